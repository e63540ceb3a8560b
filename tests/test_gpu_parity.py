"""CUDA path vs oracle, element by element, through the C ABI (needs a B200).

Integer outputs (cluster boundaries, sizes, m_i, sample rows) bit-exact; fp64
outputs within 1e-9 relative (north_star).  Inputs are seeded and synthetic
(tracegen + small hand-made edge cases); the oracle never sees GPU output."""
import numpy as np
import pytest

import oracle as O
import tracegen as G
from parity_util import Z95, assert_plans_equal

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def sr():
    import paper_conf_micro_chungnkk25_b200 as m
    m.build()
    return m


@pytest.fixture(scope="module")
def ctx(sr):
    c = sr.Context(0)
    yield c
    c.close()


def _dev(a):
    import torch
    return torch.from_numpy(np.ascontiguousarray(a).view(np.int32)).cuda()


def _both(ctx, kid, t, K, metrics=None, host=False, **kw):
    kw.setdefault("z", Z95)
    eps = kw.pop("eps", 0.05)
    if host:
        got = ctx.plan(kid, t, K, eps=eps, metrics=metrics, **kw)
    else:
        import torch
        met = None if metrics is None else torch.from_numpy(np.ascontiguousarray(metrics)).cuda()
        got = ctx.plan(_dev(kid), _dev(t), K, eps=eps, metrics=met, **kw)
    ref = O.plan(kid, t, K, eps=eps, metrics=metrics, **kw)
    return got, ref


# ------------------------------------------------------------------ pinned worked examples
def test_worked_trees(ctx, golden):
    for tr in golden("root_trees.json")["trees"]:
        t = np.array(tr["t"], np.uint32)
        got, ref = _both(ctx, np.zeros(len(t), np.uint32), t, 1, eps=tr["eps"], z=tr["z"], seed=3)
        assert_plans_equal(got, ref)
        assert [[int(c["lo_ns"]), int(c["hi_ns"])] for c in got["clusters"]] == tr["leaves_lo_hi"]
        assert got["est_total_ns"] == tr["est"]


def test_exact_tie_split(ctx, golden):
    for c in golden("split_tie.json")["cases"]:
        t = np.array([c["s"] * x for x in c["base"]] * 3, np.uint32)
        kid = np.repeat(np.arange(3, dtype=np.uint32), len(c["base"]))
        t = np.concatenate([np.sort(t[kid == k]) for k in range(3)]).astype(np.uint32)
        got, ref = _both(ctx, kid, t, 3, eps=0.05)
        assert_plans_equal(got, ref)


# ------------------------------------------------------------------ edge cases
EDGE = {
    "single_row": (np.array([0], np.uint32), np.array([5], np.uint32), 1),
    "constant": (np.zeros(1000, np.uint32), np.full(1000, 77, np.uint32), 1),
    "zeros": (np.zeros(50, np.uint32), np.zeros(50, np.uint32), 1),
    "max_t": (np.zeros(4000, np.uint32), np.where(np.arange(4000) % 3 == 0, 2 ** 32 - 1, 2 ** 31).astype(np.uint32), 1),
    "singletons_and_empty": (np.array([0, 2, 2, 5, 9, 9, 9], np.uint32), np.array([3, 1, 1, 8, 0, 4, 4], np.uint32), 12),
    "two_values": (np.zeros(9000, np.uint32), (np.arange(9000) % 2 * 1000 + 10).astype(np.uint32), 1),
    "decreasing": (np.zeros(3000, np.uint32), np.arange(3000, 0, -1).astype(np.uint32) * 1000, 1),
    "one_off_short_call": (np.zeros(5000, np.uint32), np.r_[[100], np.full(4999, 150000)].astype(np.uint32), 1),
}


@pytest.mark.parametrize("name", sorted(EDGE))
def test_edge_cases(ctx, name):
    kid, t, K = EDGE[name]
    for kw in ({}, {"root": False}, {"census_cap": True, "eps": 1e-4}):
        got, ref = _both(ctx, kid, t, K, seed=11, **kw)
        assert_plans_equal(got, ref)


def test_errors(ctx, sr):
    with pytest.raises(sr.StemError) as e:
        ctx.plan(_dev(np.array([0, 4], np.uint32)), _dev(np.array([1, 2], np.uint32)), 4)
    assert e.value.status == sr.STEM_E_RANGE
    with pytest.raises(sr.StemError) as e:
        ctx.plan(_dev(np.array([0], np.uint32)), _dev(np.array([1], np.uint32)), 1, eps=1.5)
    assert e.value.status == sr.STEM_E_INVAL
    # the context stays usable after an error
    got, ref = _both(ctx, *EDGE["two_values"][:2], 1)
    assert_plans_equal(got, ref)


# ------------------------------------------------------------------ random traces, several tiles + ragged tail
def _mixture(rng, n, K, peaks=3, spread=0.05, max_t=2 ** 24):
    kid = (rng.zipf(1.3, n) - 1) % K
    centers = rng.integers(500, max_t, (K, peaks))
    p = rng.integers(0, peaks, n)
    t = centers[kid, p] * rng.lognormal(0.0, spread, n)
    return kid.astype(np.uint32), np.minimum(t, 2 ** 32 - 1).astype(np.uint32)


@pytest.mark.parametrize("n,K", [(4097, 3), (20011, 17), (100003, 211), (250000, 1)])
@pytest.mark.parametrize("eps", [0.01, 0.05, 0.25])
def test_random_mixtures(ctx, n, K, eps):
    rng = np.random.default_rng(n + K)
    kid, t = _mixture(rng, n, K)
    got, ref = _both(ctx, kid, t, K, eps=eps, seed=n)
    assert_plans_equal(got, ref)


@pytest.mark.parametrize("opts", [dict(scope=1), dict(scope=2), dict(root=False), dict(clamp_in_split=False),
                                  dict(census_cap=True, eps=0.002), dict(seed=2 ** 63 + 12345)])
def test_option_matrix(ctx, opts):
    rng = np.random.default_rng(5)
    kid, t = _mixture(rng, 60000, 40, peaks=4, spread=0.2)
    got, ref = _both(ctx, kid, t, 40, **opts)
    assert_plans_equal(got, ref)


def test_host_pointers_and_metrics(ctx):
    rng = np.random.default_rng(9)
    kid, t = _mixture(rng, 30000, 25)
    met = np.vstack([t * 1.5 + 3, rng.random(30000)])
    got, ref = _both(ctx, kid, t, 25, metrics=met, host=True)
    assert_plans_equal(got, ref, metrics=True)
    got, ref = _both(ctx, kid, t, 25, metrics=met)
    assert_plans_equal(got, ref, metrics=True)


@pytest.mark.parametrize("host", [False, True])
@pytest.mark.parametrize("opts", [dict(), dict(root=False), dict(scope=2), dict(census_cap=True, eps=1e-5)])
def test_metric_bounds(ctx, host, opts):
    """metric_bounds (R28): true totals and bounds element by element against the
    oracle, on columns that pin the arithmetic (t itself, an affine map, a
    constant, an all-zero column, noise, a signed column)."""
    rng = np.random.default_rng(17)
    n = 50000
    kid, t = _mixture(rng, n, 30, peaks=3, spread=0.1)
    tf = t.astype(np.float64)
    met = np.vstack([tf, 2.5 * tf + 1e5, np.full(n, 3.0), np.zeros(n), rng.random(n), rng.standard_normal(n)])
    kw = dict(opts)
    kw.setdefault("eps", 0.02)
    got, ref = _both(ctx, kid, t, 30, metrics=met, host=host, metric_bounds=True, seed=8, **kw)
    assert_plans_equal(got, ref, metrics=True)
    assert got["bound_metric"][0] == pytest.approx(got["bound"], rel=1e-9)
    assert got["bound_metric"][2] == 0.0 and got["bound_metric"][3] == 0.0 and got["true_metric"][3] == 0.0
    off, _ = _both(ctx, kid, t, 30, metrics=met, host=host, seed=8, **kw)
    assert off["true_metric"] is None and off["bound_metric"] is None


def test_determinism(ctx):
    rng = np.random.default_rng(13)
    kid, t = _mixture(rng, 200000, 64)
    a = ctx.plan(_dev(kid), _dev(t), 64, z=Z95)
    b = ctx.plan(_dev(kid), _dev(t), 64, z=Z95)
    assert a["clusters"].tobytes() == b["clusters"].tobytes()
    assert a["sample_row"].tobytes() == b["sample_row"].tobytes()
    assert a["est_total_ns"] == b["est_total_ns"] and a["bound"] == b["bound"]


def test_z_from_conf_matches_scipy(sr):
    from scipy.stats import norm
    for conf in (0.8, 0.9, 0.95, 0.99, 0.999999):
        assert sr.z_from_conf(conf) == pytest.approx(norm.isf((1 - conf) / 2), rel=1e-14)


# ------------------------------------------------------------------ config-shaped traces (BASELINE configs)
@pytest.mark.parametrize("name,n", [("C1", None), ("C2", None), ("C4", 2_000_000)])
def test_configs(ctx, name, n):
    sp = G.spec(name, n=n)
    kid, t, _ = G.generate_np(sp)
    got, ref = _both(ctx, kid, t, sp.n_kernels, eps=sp.eps, seed=1)
    assert_plans_equal(got, ref)


def test_config_c3_with_metrics(ctx):
    sp = G.spec("C3", n=2_000_000)
    kid, t, met = G.generate_np(sp)
    got, ref = _both(ctx, kid, t, sp.n_kernels, metrics=met, eps=sp.eps, seed=2, metric_bounds=True)
    assert_plans_equal(got, ref, metrics=True)


@pytest.mark.parametrize("eps", [0.01, 0.03, 0.1])
def test_eps_sweep(ctx, eps):
    sp = G.spec("C4", n=1_000_000)
    kid, t, _ = G.generate_np(sp)
    got, ref = _both(ctx, kid, t, sp.n_kernels, eps=eps, seed=4)
    assert_plans_equal(got, ref)


# ------------------------------------------------------------------ generator twin
def test_tracegen_cuda_matches_numpy():
    import torch
    for name, n, row0 in (("C3", 300_000, 12_345_677), ("C2", 100_000, 0), ("C1", 10_000, 0)):
        sp = G.spec(name)
        ds = G.DeviceSpec(sp, "cuda:0")
        k = torch.empty(n, dtype=torch.int32, device="cuda")
        tt = torch.empty(n, dtype=torch.int32, device="cuda")
        met = torch.empty((sp.n_metrics, n), dtype=torch.float64, device="cuda") if sp.n_metrics else None
        G.generate_cuda(ds, k, tt, met, row0=row0, count=n)
        kid, t, m = G.generate_np(sp, row0, n)
        assert np.array_equal(k.cpu().numpy().view(np.uint32), kid)
        assert np.array_equal(tt.cpu().numpy().view(np.uint32), t)
        if sp.n_metrics:
            assert np.array_equal(met.cpu().numpy(), m)


# ------------------------------------------------------------------ full BASELINE sizes
def test_config_c3_full_size_with_metrics(ctx):
    """configs[2] at its full size (20M rows, 12 metric columns), host-pointer path
    (the e2e launch), element by element against the oracle."""
    sp = G.spec("C3")
    kid, t, met = G.generate_np(sp)
    got, ref = _both(ctx, kid, t, sp.n_kernels, metrics=met, host=True, eps=sp.eps, seed=12345, metric_bounds=True)
    assert_plans_equal(got, ref, metrics=True)


@pytest.mark.slow
@pytest.mark.parametrize("split", [0, 1, 2])
def test_config_c5_full_size_sampled(ctx, split):
    """configs[4] (1e9 rows, 10k kernels) in the launch configuration bench.py times:
    device-resident trace, default options (and the two Lloyd split rules, R26/R27,
    as `bench.py --split` runs them).  The oracle recomputes the ROOT leaves of
    sampled kernels one by one (leaves of a kernel depend only on its rows);
    global outputs are checked through properties that hold at any size."""
    import torch
    sp = G.spec("C5")
    ds = G.DeviceSpec(sp, "cuda:0")
    kid = torch.empty(sp.n, dtype=torch.int32, device="cuda")
    tt = torch.empty(sp.n, dtype=torch.int32, device="cuda")
    G.generate_cuda(ds, kid, tt)
    p = ctx.plan(kid, tt, sp.n_kernels, eps=sp.eps, z=Z95, seed=12345, split=split)
    cl = p["clusters"]
    # properties: partition, exact total, ordering, bound, samples inside their clusters
    counts = torch.bincount(kid, minlength=sp.n_kernels).cpu().numpy()
    per_kernel = np.bincount(cl["kernel_id"], weights=cl["n"], minlength=sp.n_kernels)
    assert np.array_equal(per_kernel.astype(np.int64), counts.astype(np.int64))
    tot = int((tt.to(torch.int64) & 0xFFFFFFFF).sum().item())
    assert p["true_total_ns"] == tot == int(cl["sum_ns"].astype(object).sum())
    assert np.all(np.diff(cl["kernel_id"].astype(np.int64)) >= 0)
    assert p["bound"] <= sp.eps and np.all(cl["m"] >= 1)
    rows = torch.from_numpy(p["sample_row"].astype(np.int64)).cuda()
    sc = p["sample_cluster"]
    t_s = (tt[rows].to(torch.int64) & 0xFFFFFFFF).cpu().numpy()
    k_s = kid[rows].cpu().numpy()
    assert np.array_equal(k_s, cl["kernel_id"][sc].astype(np.int32))
    assert np.all((t_s >= cl["lo_ns"][sc]) & (t_s <= cl["hi_ns"][sc]))
    # element-wise: the oracle's leaves of sampled kernels (small to mid-size groups)
    rng = np.random.default_rng(7)
    cand = np.nonzero((counts > 1000) & (counts < 3_000_000))[0]
    for k in list(rng.choice(cand, 6, replace=False)) + [int(np.argmin(np.where(counts > 0, counts, 1 << 40)))]:
        sel = torch.nonzero(kid == int(k)).flatten()
        sub_t = (tt[sel].to(torch.int64) & 0xFFFFFFFF).cpu().numpy().astype(np.uint32)
        ref = O.plan(np.zeros(len(sub_t), np.uint32), sub_t, 1, eps=sp.eps, z=Z95, seed=12345, split=split)
        mine = cl[cl["kernel_id"] == k]
        for f in ("ordinal", "lo_ns", "hi_ns", "n", "sum_ns"):
            assert np.array_equal(mine[f].astype(np.int64), ref[f].astype(np.int64)), (k, f)


# ------------------------------------------------------------------ big clusters (chunk-bound path, >= 65536 rows)
BIG = {
    "distinct_ramp": lambda: np.arange(300_000, dtype=np.uint32) * 7 + 1000,
    "two_values_outlier": lambda: np.r_[np.full(150_000, 5), np.full(120_000, 6), [4000]].astype(np.uint32),
    "symmetric_tie": lambda: np.r_[np.full(70_000, 0), np.full(90_000, 10), np.full(70_000, 20)].astype(np.uint32),
    "lognormal_wide": lambda: (np.random.default_rng(3).lognormal(12, 1.1, 500_000)).astype(np.uint32),
    "near_constant": lambda: (3_000_000_000 + np.random.default_rng(4).integers(0, 3, 200_000)).astype(np.uint32),
}


@pytest.mark.parametrize("name", sorted(BIG))
def test_big_clusters(ctx, name):
    t = BIG[name]()
    rng = np.random.default_rng(len(t))
    perm = rng.permutation(len(t))
    kid = np.zeros(len(t), np.uint32)
    got, ref = _both(ctx, kid, t[perm], 1, eps=0.02, seed=4)
    assert_plans_equal(got, ref)


# ------------------------------------------------------------------ sort modes (sort.cu): row payload vs packed key
def _dup_heavy(n, K, seed):
    """few distinct times per kernel: long runs of equal (kernel, t), the case
    where a packed key's low row bits match several candidate rows"""
    rng = np.random.default_rng(seed)
    kid = rng.integers(0, K, n).astype(np.uint32)
    base = rng.integers(1000, 50_000, K)
    t = base[kid] + rng.integers(0, 6, n) * (base[kid] // 7)
    return kid, t.astype(np.uint32)


@pytest.mark.parametrize("mode", ["payload", "packed", "bits16", "bits12"])
@pytest.mark.parametrize("eps", [0.002, 0.05])
def test_sort_modes(ctx, monkeypatch, mode, eps):
    """Every sort mode gives the oracle's plan bit for bit; the forced small
    packings (4 and 49 candidate rows per sample) go through the ambiguous-run
    resolution, which the default packing at these sizes never needs."""
    if mode == "payload":
        monkeypatch.setenv("STEMROOT_SORT_PACK", "0")
    elif mode.startswith("bits"):
        monkeypatch.setenv("STEMROOT_PACK_BITS", mode[4:])
    kid, t = _dup_heavy(200_003, 7, 17)
    got, ref = _both(ctx, kid, t, 7, eps=eps, seed=21)
    assert_plans_equal(got, ref)
    st = ctx.stats()
    assert st["pack_bits"] == {"payload": 0, "bits16": 16, "bits12": 12}.get(mode, st["key_bits"] and 64 - st["key_bits"])
    if mode.startswith("bits") and eps == 0.002:
        assert st["ambiguous_samples"] > 0



@pytest.mark.parametrize("rank", ["match", "ballot"])
@pytest.mark.parametrize("pack", ["0", "1"])
def test_sort_ranking_modes(ctx, monkeypatch, rank, pack):
    """each warp ranking method of the radix passes (match.any, 8 ballots)
    in both key layouts gives the oracle's plan"""
    monkeypatch.setenv("STEMROOT_SORT_RANK", rank)
    monkeypatch.setenv("STEMROOT_SORT_PACK", pack)
    rng = np.random.default_rng(99)
    kid, t = _mixture(rng, 150_001, 300, peaks=3, spread=0.3)
    got, ref = _both(ctx, kid, t, 300, eps=0.03, seed=5)
    assert_plans_equal(got, ref)


@pytest.mark.parametrize("coarse", ["0", "1"])
@pytest.mark.parametrize("K", [3, 700])
def test_key_bases_heavy_tails(ctx, sr, monkeypatch, coarse, K):
    """fine (2^16) and coarse (2^24) kernel key bases; heavy tails put many
    rows at t >= 2^24, which the coarse pass histograms take from the
    per-kernel tail histogram of the pre-pass"""
    monkeypatch.setenv("STEMROOT_SORT_COARSE", coarse)
    rng = np.random.default_rng(K)
    n = 300_007
    kid = rng.integers(0, K, n).astype(np.uint32)
    t = np.minimum(rng.lognormal(14 + (kid % 5), 1.6, n), 2 ** 32 - 1).astype(np.uint32)
    t[::997] = 2 ** 32 - 1
    got, ref = _both(ctx, kid, t, K, eps=0.05, seed=3)
    assert_plans_equal(got, ref)
    assert ctx.stats()["coarse_bases"] == (1 if coarse == "1" else 0)


def test_big_path_multi_segment(ctx):
    """The big-cluster path on clusters spanning many 65536-row blocks, starting at
    unaligned rows, with ties and constant runs, against the oracle."""
    rng = np.random.default_rng(11)
    parts = [
        (0, rng.integers(0, 5, 1_234) + 100),                                    # unaligns the next group
        (1, rng.lognormal(11, 1.0, 2_500_000)),                                  # heavy tail
        (2, np.r_[np.full(400_000, 5000), np.full(700_001, 9000), rng.integers(20_000, 20_003, 300_000)]),
        (3, rng.normal(50_000, 2_000, 1_100_000).clip(1)),                       # unimodal, wide plateau
    ]
    kid = np.concatenate([np.full(len(p), k, np.uint32) for k, p in parts])
    t = np.concatenate([np.asarray(p) for _, p in parts]).astype(np.uint32)
    perm = rng.permutation(len(t))
    got, ref = _both(ctx, kid[perm], t[perm], 4, eps=0.01, seed=8)
    assert_plans_equal(got, ref)


@pytest.mark.parametrize("n", [1, 31, 32, 33, 16352, 16353, 16384, 16385, 65536 * 2 + 7])
def test_tile_boundaries(ctx, n):
    """sizes at the 32-row chunk, the 16 384-row prefix-moment tile (the scan
    element past the last chunk opening a tile of its own), the 65 536-row
    leaf-bitmap tile and the 5120-row sort tile boundaries"""
    rng = np.random.default_rng(n)
    kid, t = _mixture(rng, n, 3 if n > 3 else 1, peaks=2, spread=0.2)
    got, ref = _both(ctx, kid, t, 3 if n > 3 else 1, eps=0.02, seed=n)
    assert_plans_equal(got, ref)


# ------------------------------------------------------------------ split variant: Lloyd's k-means (R26)
@pytest.mark.parametrize("case", ["mixture", "c2", "big", "ties"])
def test_lloyd_split_variant(ctx, case):
    """opts.split = 1 (Lloyd's k-means, k = 2, from (min, max), P:L192/P:L258,
    reading R26): clusters, sizes and sample rows bit-exact against the oracle's
    step-by-step Lloyd, on mixtures, a CASIO-shaped trace, multi-block clusters
    and long runs of equal times."""
    rng = np.random.default_rng(5)
    if case == "mixture":
        kid, t = _mixture(rng, 150_001, 97, peaks=4, spread=0.3)
        K = 97
    elif case == "c2":
        sp = G.spec("C2", n=300_000)
        kid, t, _ = G.generate_np(sp)
        K = sp.n_kernels
    elif case == "big":
        t = np.concatenate([rng.lognormal(11, 1.0, 700_000), rng.normal(5e4, 3e3, 400_000).clip(1)]).astype(np.uint32)
        kid = np.r_[np.zeros(700_000, np.uint32), np.ones(400_000, np.uint32)]
        K = 2
    else:
        kid, t = _dup_heavy(200_003, 7, 3)
        K = 7
    got, ref = _both(ctx, kid, t, K, eps=0.03, seed=9, split=1)
    assert_plans_equal(got, ref)
    # the variant is a different rule: the default's leaves differ somewhere
    if case in ("mixture", "c2"):
        d = O.plan(kid, t, K, eps=0.03, z=Z95, seed=9)
        assert len(d["n"]) != len(ref["n"]) or not np.array_equal(d["n"], ref["n"])


# ------------------------------------------------------------------ split variant: k-means++ seeded Lloyd (R27)
@pytest.mark.parametrize("case", ["mixture", "c2", "big", "ties"])
def test_kmpp_split_variant(ctx, case):
    """opts.split = 2 (Lloyd's k-means, k = 2, from k-means++ seeds drawn with
    Philox on (min t, max t, n) keyed by the seed, reading R27): clusters,
    sizes and sample rows bit-exact against the oracle's step-by-step seeding
    and Lloyd iteration, for two seeds (the trees differ between them)."""
    rng = np.random.default_rng(6)
    if case == "mixture":
        kid, t = _mixture(rng, 150_001, 97, peaks=4, spread=0.3)
        K = 97
    elif case == "c2":
        sp = G.spec("C2", n=300_000)
        kid, t, _ = G.generate_np(sp)
        K = sp.n_kernels
    elif case == "big":
        t = np.concatenate([rng.lognormal(11, 1.0, 700_000), rng.normal(5e4, 3e3, 400_000).clip(1)]).astype(np.uint32)
        kid = np.r_[np.zeros(700_000, np.uint32), np.ones(400_000, np.uint32)]
        K = 2
    else:
        kid, t = _dup_heavy(200_003, 7, 3)
        K = 7
    refs = []
    for seed in (9, 0xDEADBEEFCAFEF00D):
        got, ref = _both(ctx, kid, t, K, eps=0.03, seed=seed, split=2)
        assert_plans_equal(got, ref)
        refs.append(ref)
    if case in ("mixture", "c2"):
        a, b = refs
        assert len(a["n"]) != len(b["n"]) or not np.array_equal(a["n"], b["n"])


def test_split_option_validation(ctx, sr):
    kid = np.zeros(100, np.uint32)
    t = np.arange(100, dtype=np.uint32)
    with pytest.raises(sr.StemError):
        ctx.plan(kid, t, 1, split=4)
    with pytest.raises(sr.StemError):
        ctx.plan(kid, t, 1, split=-1)
    for k in (0, 1, 9):
        with pytest.raises(sr.StemError):
            ctx.plan(kid, t, 1, split=3, kmeans_k=k)


# ------------------------------------------------------------------ split variant: exact k-means, k > 2 (R29)
def _few_values(rng, n, K, vals=150):
    """mixtures whose kernels have at most `vals` distinct times (the oracle's
    exact DP is O(k d^2) in the distinct values d)"""
    kid = rng.integers(0, K, n).astype(np.uint32)
    base = rng.integers(2000, 200_000, (K, 3))
    peak = rng.integers(0, 3, n)
    q = rng.integers(0, vals // 3, n)
    t = base[kid, peak] + q * (base[kid, 0] // 400 + 1)
    return kid, t.astype(np.uint32)


@pytest.mark.parametrize("k", [2, 3, 4, 8])
@pytest.mark.parametrize("case", ["mixture", "ties", "big"])
def test_kmeans_split_variant(ctx, k, case):
    rng = np.random.default_rng(k * 7 + len(case))
    if case == "mixture":
        kid, t = _few_values(rng, 40_000, 12)
        K = 12
    elif case == "ties":   # evenly spaced values: many optimal partitions, the tie rule decides
        kid = rng.integers(0, 3, 9000).astype(np.uint32)
        t = (rng.integers(0, 12, 9000) * 100 + 1000 + kid * 5000).astype(np.uint32)
        K = 3
    else:                  # one kernel, 300k rows over ~300 values (many D&C rounds, big frontier clusters)
        kid = np.zeros(300_000, np.uint32)
        t = (np.round(rng.lognormal(5, 0.4, 300_000)) * 3).astype(np.uint32)
        K = 1
    for eps in (0.01, 0.05):
        got, ref = _both(ctx, kid, t, K, eps=eps, seed=9, split=3, kmeans_k=k)
        assert_plans_equal(got, ref)
    if k == 2:   # k = 2 is the default exact 2-means (R5)
        a = ctx.plan(_dev(kid), _dev(t), K, z=Z95, seed=9, split=3, kmeans_k=2)
        b = ctx.plan(_dev(kid), _dev(t), K, z=Z95, seed=9)
        assert a["clusters"].tobytes() == b["clusters"].tobytes()


@pytest.mark.parametrize("split", [0, 1, 2])
def test_pipelined_levels_match_synchronous(ctx, monkeypatch, split):
    """the pipelined ROOT level loop (the next level queued before the host sees
    the frontier size) gives the same plan as one host round trip per level"""
    rng = np.random.default_rng(77)
    kid, t = _mixture(rng, 120_011, 41, peaks=5, spread=0.4)
    a = ctx.plan(kid, t, 41, eps=0.02, z=Z95, seed=2, split=split)
    monkeypatch.setenv("STEMROOT_LEVEL_SYNC", "1")
    b = ctx.plan(kid, t, 41, eps=0.02, z=Z95, seed=2, split=split)
    for f in ("kernel_id", "ordinal", "lo_ns", "hi_ns", "n", "sum_ns", "m"):
        assert np.array_equal(a["clusters"][f], b["clusters"][f]), f
    assert np.array_equal(a["sample_row"], b["sample_row"])
    assert a["est_total_ns"] == b["est_total_ns"]


@pytest.mark.parametrize("s32", ["0", "1"])
def test_sort_status_widths(ctx, monkeypatch, s32):
    """32-bit look-back statuses (n < 2^30, the default) and the 64-bit ones
    (larger traces) give the oracle's plan"""
    monkeypatch.setenv("STEMROOT_SORT_S32", s32)
    rng = np.random.default_rng(31)
    kid, t = _mixture(rng, 400_009, 123, peaks=3, spread=0.3)
    got, ref = _both(ctx, kid, t, 123, eps=0.03, seed=12)
    assert_plans_equal(got, ref)


def test_local_subtree_path_all_split_rules(tmp_path):
    """STEMROOT_LOCAL_ROWS (the optional local subtree kernel, exact split only;
    read once per process, hence the subprocess) gives the oracle's plan with
    every split rule: the Lloyd rules keep all clusters on the level path."""
    import os
    import subprocess
    import sys
    here = os.path.dirname(os.path.abspath(__file__))
    root = os.path.dirname(here)
    script = tmp_path / "local.py"
    script.write_text(f"""
import sys
sys.path[:0] = [{root!r}, {here!r}]
import numpy as np, torch
import oracle as O, tracegen as G
import paper_conf_micro_chungnkk25_b200 as sr
from parity_util import Z95, assert_plans_equal
sp = G.spec("C2", n=200_000)
kid, t, _ = G.generate_np(sp)
ctx = sr.Context(0)
for split in (0, 1, 2):
    got = ctx.plan(torch.from_numpy(kid.view(np.int32)).cuda(), torch.from_numpy(t.view(np.int32)).cuda(),
                   sp.n_kernels, eps=0.03, z=Z95, seed=5, split=split)
    ref = O.plan(kid, t, sp.n_kernels, eps=0.03, z=Z95, seed=5, split=split)
    assert_plans_equal(got, ref)
print("ok")
""")
    env = dict(os.environ, STEMROOT_LOCAL_ROWS="1024")
    out = subprocess.run([sys.executable, str(script)], env=env, capture_output=True, text=True, timeout=300)
    assert out.returncode == 0 and out.stdout.strip().endswith("ok"), out.stdout[-2000:] + out.stderr[-2000:]


def test_metric_bounds_trace_order_path(tmp_path):
    """metric_bounds has two GPU paths: sorted order (one GPU, every sorted
    position's row known: the default above) and trace order with per-leaf
    atomics (multi-GPU and multi-candidate packed keys); STEMROOT_MB_TRACE_ORDER
    forces the latter on one GPU.  Both match the oracle."""
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    prog = tmp_path / "mb.py"
    prog.write_text(
        "import sys, numpy as np, torch\n"
        f"sys.path.insert(0, {root!r}); sys.path.insert(0, {os.path.join(root, 'tests')!r})\n"
        "import paper_conf_micro_chungnkk25_b200 as sr, oracle as O, tracegen as G\n"
        "from parity_util import Z95, assert_plans_equal\n"
        "sp = G.spec('C3', n=300_000); kid, t, met = G.generate_np(sp)\n"
        "ctx = sr.Context(0)\n"
        "got = ctx.plan(kid, t, sp.n_kernels, metrics=met, eps=0.02, z=Z95, seed=3, metric_bounds=True)\n"
        "ref = O.plan(kid, t, sp.n_kernels, metrics=met, eps=0.02, z=Z95, seed=3, metric_bounds=1)\n"
        "assert_plans_equal(got, ref, metrics=True); print('MB_OK')\n")
    out = subprocess.run([sys.executable, str(prog)], env=dict(os.environ, STEMROOT_MB_TRACE_ORDER="1"),
                         capture_output=True, text=True, timeout=600)
    assert "MB_OK" in out.stdout, out.stdout + out.stderr[-3000:]


@pytest.mark.parametrize("opts", [dict(scope=1), dict(scope=2), dict(census_cap=True, eps=1e-4),
                                  dict(clamp_in_split=False)])
def test_kmeans_option_matrix(ctx, opts):
    rng = np.random.default_rng(71)
    kid, t = _few_values(rng, 20_000, 6)
    kw = dict(opts)
    kw.setdefault("eps", 0.02)
    got, ref = _both(ctx, kid, t, 6, seed=5, split=3, kmeans_k=3, **kw)
    assert_plans_equal(got, ref)


# ------------------------------------------------------------------ value-histogram ROOT (root.cu DensePath, VrRun)
def _value_case(case, seed):
    rng = np.random.default_rng(seed)
    if case == "dup_heavy":
        return _dup_heavy(400_000, 37, seed) + (37,)
    K = 23
    kid, t = _mixture(rng, 300_001, K, peaks=4, spread=0.3, max_t=2 ** 22)
    if case == "quantised":     # microsecond timer: long runs of equal times
        t = (t // 1000 * 1000 + 1000).astype(np.uint32)
    elif case == "mixed":       # even kernels quantised, odd ones continuous
        q = kid % 2 == 0
        t[q] = t[q] // 5000 * 5000 + 7
    elif case == "two_values":  # one kernel of two times and an outlier, the rest continuous
        t[kid == 0] = np.where(rng.random(int((kid == 0).sum())) < 0.6, 4000, 4001)
        t[np.flatnonzero(kid == 0)[:1]] = 900_000
    return kid, t.astype(np.uint32), K


@pytest.mark.parametrize("min_rows", ["64", "4096", "0"])
@pytest.mark.parametrize("case", ["dup_heavy", "quantised", "mixed", "two_values"])
def test_value_path_matches_oracle(ctx, monkeypatch, min_rows, case):
    """Groups whose times repeat take the value-histogram ROOT (their tree built
    over distinct values on a side stream, beside the row levels);
    STEMROOT_VALUE_ROWS is the group size from which a group is tested, 0 turns
    the path off.  The plan equals the oracle's either way."""
    kid, t, K = _value_case(case, 3)
    monkeypatch.setenv("STEMROOT_VALUE_ROWS", min_rows)
    got, ref = _both(ctx, kid, t, K, eps=0.01, seed=6)
    assert_plans_equal(got, ref)
    st = ctx.stats()
    if min_rows == "0":
        assert st["value_groups"] == 0 and st["value_levels"] == 0
    elif case in ("dup_heavy", "quantised"):
        assert st["value_groups"] > 0 and 0 < st["value_count"] < len(t) // 4
        assert st["value_levels"] > 0


@pytest.mark.parametrize("ratio", ["2", "64"])
@pytest.mark.parametrize("opts", [dict(), dict(scope=2), dict(census_cap=True, eps=0.002), dict(clamp_in_split=False)])
def test_value_path_options(ctx, monkeypatch, ratio, opts):
    kid, t, K = _value_case("mixed", 9)
    monkeypatch.setenv("STEMROOT_VALUE_ROWS", "256")
    monkeypatch.setenv("STEMROOT_VALUE_RATIO", ratio)
    kw = dict(seed=2)
    kw.update(opts)
    eps = kw.pop("eps", 0.02)
    got, ref = _both(ctx, kid, t, K, eps=eps, **kw)
    assert_plans_equal(got, ref)


def test_value_path_active_rows_and_levels(ctx, monkeypatch):
    """the value path reports the same ROOT work as the row levels: the rows of
    every cluster it decides (active_rows) and the tree depth"""
    kid, t, K = _value_case("quantised", 4)
    monkeypatch.setenv("STEMROOT_VALUE_ROWS", "0")
    ctx.plan(_dev(kid), _dev(t), K, eps=0.01, z=Z95, seed=1)
    rows_path = ctx.stats()
    monkeypatch.setenv("STEMROOT_VALUE_ROWS", "64")
    ctx.plan(_dev(kid), _dev(t), K, eps=0.01, z=Z95, seed=1)
    val_path = ctx.stats()
    assert val_path["value_groups"] > 0
    assert val_path["active_rows"] == rows_path["active_rows"]
    assert max(val_path["levels"], val_path["value_levels"]) == rows_path["levels"]


# ------------------------------------------------------------------ nearest-centre descent (root.cu nc_split_kernel)
def _nc_case(case):
    if case in BIG:
        t = BIG[case]()
        perm = np.random.default_rng(len(t)).permutation(len(t))
        return np.zeros(len(t), np.uint32), t[perm], 1, 0.02
    if case in EDGE:
        kid, t, K = EDGE[case]
        return kid, t, K, 0.05
    if case == "mixture":
        kid, t = _mixture(np.random.default_rng(11), 250_000, 19, peaks=5, spread=0.1)
        return kid, t, 19, 0.01
    if case == "dup_heavy":
        return _dup_heavy(300_000, 29, 5) + (29, 0.005)
    if case in ("quantised", "two_values"):
        return _value_case(case, 7) + (0.01,)
    sp = G.spec(case, n=1_500_000 if case == "C3" else None)
    kid, t, _ = G.generate_np(sp)
    return kid, t, sp.n_kernels, sp.eps


@pytest.mark.parametrize("nc", ["0", "1", "2"])
@pytest.mark.parametrize("case", sorted(BIG) + ["two_values", "one_off_short_call", "max_t", "mixture", "dup_heavy",
                                                "quantised", "C2", "C3"])
def test_nearest_centre_descent(ctx, monkeypatch, nc, case):
    """The exact split by the nearest-centre descent (STEMROOT_SPLIT_NC=2, the
    default: every cluster; 1: big clusters, chunk bounds for the rest; 0: the
    chunk-bound kernels alone) equals the oracle's tree, samples and estimate
    (the value path off, so every group takes the row levels)."""
    kid, t, K, eps = _nc_case(case)
    monkeypatch.setenv("STEMROOT_SPLIT_NC", nc)
    monkeypatch.setenv("STEMROOT_VALUE_ROWS", "0")
    got, ref = _both(ctx, kid, t, K, eps=eps, seed=3)
    assert_plans_equal(got, ref)


def test_nearest_centre_descent_ties(ctx, monkeypatch, golden):
    monkeypatch.setenv("STEMROOT_SPLIT_NC", "2")
    test_exact_tie_split(ctx, golden)
    test_worked_trees(ctx, golden)


def test_host_trace_chunked_copy(ctx):
    """A host trace of >= 2^24 rows is copied in chunks, each consumed by the
    pre-pass as it lands (sort.cu h2d_chunks): the plan equals the oracle's."""
    sp = G.spec("C4", n=(1 << 24) + 4099)
    kid, t, _ = G.generate_np(sp)
    got, ref = _both(ctx, kid, t, sp.n_kernels, host=True, eps=sp.eps, seed=5)
    assert_plans_equal(got, ref)


@pytest.mark.parametrize("K", [30_000, 100_000])
def test_many_kernel_ids(ctx, K):
    """More kernel ids than the pre-pass keeps in shared memory (> 24 000: global
    count/max atomics) and than the coarse key bases allow (> 65 536); ids used
    sparsely, several tiles and a ragged tail"""
    rng = np.random.default_rng(K)
    n = 400_003
    kid = (rng.zipf(1.2, n) * 7919 % K).astype(np.uint32)
    t = (rng.lognormal(9, 0.8, n) * (1 + kid % 13)).astype(np.uint32)
    got, ref = _both(ctx, kid, t, K, eps=0.05, seed=8)
    assert_plans_equal(got, ref)
