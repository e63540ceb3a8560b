"""Multi-GPU path on one B200: world ranks emulated by threads
sharing cuda:0 through the loopback communicator (the same C++ SPMD code the
NCCL communicator drives), and a real one-rank NCCL communicator.  The
gathered plan must equal the single-GPU plan: integers bit-exact, fp64 sums
within 1e-9 relative (their summation order depends on the rank count)."""
import os
import threading

import numpy as np
import pytest

import oracle as O
import tracegen as G
from parity_util import Z95, assert_plans_equal

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def sr():
    import paper_conf_micro_chungnkk25_b200 as m
    m.build()
    return m


def _dist_plan(sr, kid, t, K, world, metrics=None, stats_out=None, **kw):
    import torch
    n = len(kid)
    cuts = [n * r // world for r in range(world + 1)]
    comms = sr.Comm.loopback(world, 0)
    ctxs = [sr.Context(0) for _ in range(world)]
    streams = [torch.cuda.Stream() for _ in range(world)]
    shards = []
    for r in range(world):
        a, b = cuts[r], cuts[r + 1]
        dk = torch.from_numpy(np.ascontiguousarray(kid[a:b]).view(np.int32)).cuda()
        dt = torch.from_numpy(np.ascontiguousarray(t[a:b]).view(np.int32)).cuda()
        dm = None if metrics is None else torch.from_numpy(np.ascontiguousarray(metrics[:, a:b])).cuda()
        shards.append((dk, dt, dm))
    torch.cuda.synchronize()
    out, err = [None] * world, [None] * world

    def run(r):
        try:
            dk, dt, dm = shards[r]
            out[r] = ctxs[r].plan_dist(comms[r], dk, dt, K, cuts[r], metrics=dm, stream=streams[r].cuda_stream,
                                       **kw)
        except Exception as e:  # noqa: BLE001
            err[r] = e
    th = [threading.Thread(target=run, args=(r,)) for r in range(world)]
    for x in th:
        x.start()
    for x in th:
        x.join(timeout=600)
    for e in err:
        if e is not None:
            raise e
    assert all(o is None for o in out[1:])
    if stats_out is not None:
        stats_out.extend(c.stats() for c in ctxs)
    for c in ctxs:
        c.close()
    for c in comms:
        c.close()
    return out[0]


@pytest.mark.parametrize("world", [1, 2, 3, 4])
def test_loopback_matches_single_gpu(sr, world):
    sp = G.spec("C2", n=300_000)
    kid, t, _ = G.generate_np(sp)
    ref = O.plan(kid, t, sp.n_kernels, eps=0.05, z=Z95, seed=5)
    got = _dist_plan(sr, kid, t, sp.n_kernels, world, eps=0.05, z=Z95, seed=5)
    assert_plans_equal(got, ref)


@pytest.mark.parametrize("opts", [dict(scope=1), dict(scope=2), dict(root=False), dict(census_cap=True, eps=0.003)])
def test_loopback_options(sr, opts):
    rng = np.random.default_rng(3)
    n, K = 80_000, 37
    kid = (rng.zipf(1.3, n) % K).astype(np.uint32)
    t = (rng.integers(1, 5, K)[kid] * 10000 * rng.lognormal(0, 0.2, n)).astype(np.uint32)
    kw = dict(z=Z95, seed=9)
    kw.update(opts)
    eps = kw.pop("eps", 0.05)
    ref = O.plan(kid, t, K, eps=eps, **kw)
    got = _dist_plan(sr, kid, t, K, 3, eps=eps, **kw)
    assert_plans_equal(got, ref)


def test_loopback_metrics_and_empty_ranks(sr):
    sp = G.spec("C3", n=200_000)
    kid, t, met = G.generate_np(sp)
    ref = O.plan(kid, t, sp.n_kernels, eps=0.05, z=Z95, seed=1, metrics=met)
    got = _dist_plan(sr, kid, t, sp.n_kernels, 4, metrics=met, eps=0.05, z=Z95, seed=1)
    assert_plans_equal(got, ref, metrics=True)
    # a single kernel: ranks 1.. own no kernels and receive no rows
    kid1 = np.zeros(5000, np.uint32)
    t1 = (np.arange(5000) % 7 * 1000 + 5).astype(np.uint32)
    ref = O.plan(kid1, t1, 1, z=Z95)
    got = _dist_plan(sr, kid1, t1, 1, 3, z=Z95)
    assert_plans_equal(got, ref)


@pytest.mark.parametrize("world", [2, 4])
def test_loopback_metric_bounds(sr, world):
    """metric_bounds (R28) across ranks: every rank's leaves are gathered, each
    rank reads its home rows' metrics, the per-leaf sums are allreduced; the
    totals and bounds match the single-trace oracle"""
    sp = G.spec("C3", n=150_000)
    kid, t, met = G.generate_np(sp)
    ref = O.plan(kid, t, sp.n_kernels, eps=0.03, z=Z95, seed=5, metrics=met, metric_bounds=1)
    got = _dist_plan(sr, kid, t, sp.n_kernels, world, metrics=met, eps=0.03, z=Z95, seed=5, metric_bounds=True)
    assert_plans_equal(got, ref, metrics=True)


def _giant_trace(n, K, share, seed):
    """one kernel holding `share` of the rows (a multi-modal time mix, so its
    ROOT tree is deep), the rest spread over K - 1 small kernels"""
    rng = np.random.default_rng(seed)
    kid = np.where(rng.random(n) < share, 0, rng.integers(1, K, n)).astype(np.uint32)
    modes = np.array([20_000, 55_000, 140_000, 400_000])
    t = np.where(kid == 0, modes[rng.integers(0, 4, n)] * rng.lognormal(0, 0.15, n),
                 (kid * 3000 + 5000) * rng.lognormal(0, 0.3, n)).astype(np.uint32)
    return kid, t


@pytest.mark.parametrize("world", [2, 3, 4, 8])
def test_loopback_giant_kernel_is_split_across_ranks(sr, world):
    """A kernel larger than a rank's share (70 % of the rows): its ROOT tree is
    built on the merged value histogram and its leaves are dealt to ranks as
    units (dist.cu giant_plan).  The plan equals the single-trace oracle's
    bit-for-bit on integers, and the busiest rank owns far fewer rows than the
    70 % it would own with whole kernels."""
    n, K = 240_000, 41
    kid, t = _giant_trace(n, K, 0.7, 11 + world)
    ref = O.plan(kid, t, K, eps=0.02, z=Z95, seed=3)
    st = []
    got = _dist_plan(sr, kid, t, K, world, stats_out=st, eps=0.02, z=Z95, seed=3)
    assert_plans_equal(got, ref)
    owned = [s["owned_rows"] for s in st]
    assert sum(owned) == n
    assert max(owned) < 0.7 * n * 0.9, owned


@pytest.mark.parametrize("opts", [dict(scope=2), dict(census_cap=True, eps=0.005), dict(clamp_in_split=False)])
def test_loopback_giant_kernel_options(sr, opts):
    n, K = 120_000, 9
    kid, t = _giant_trace(n, K, 0.8, 5)
    kw = dict(z=Z95, seed=4)
    kw.update(opts)
    eps = kw.pop("eps", 0.03)
    ref = O.plan(kid, t, K, eps=eps, **kw)
    got = _dist_plan(sr, kid, t, K, 3, eps=eps, **kw)
    assert_plans_equal(got, ref)


def test_loopback_giant_kernel_with_metrics(sr):
    n, K = 100_000, 13
    kid, t = _giant_trace(n, K, 0.6, 8)
    met = np.random.default_rng(2).normal(5, 1, (2, n))
    ref = O.plan(kid, t, K, eps=0.03, z=Z95, seed=6, metrics=met, metric_bounds=1)
    got = _dist_plan(sr, kid, t, K, 4, metrics=met, eps=0.03, z=Z95, seed=6, metric_bounds=True)
    assert_plans_equal(got, ref, metrics=True)


def test_loopback_giant_kernel_disabled_by_env(sr, monkeypatch):
    """STEMROOT_DIST_GIANT=0 keeps whole kernels (the value is read once per
    process, so this runs in a child)"""
    import subprocess
    import sys
    code = (
        "import sys; sys.path.insert(0, 'tests'); sys.path.insert(0, '.')\n"
        "import numpy as np, test_gpu_dist as T, paper_conf_micro_chungnkk25_b200 as sr, oracle as O\n"
        "kid, t = T._giant_trace(60000, 7, 0.7, 1); st = []\n"
        "got = T._dist_plan(sr, kid, t, 7, 2, stats_out=st, z=T.Z95)\n"
        "T.assert_plans_equal(got, O.plan(kid, t, 7, z=T.Z95))\n"
        "assert max(s['owned_rows'] for s in st) >= 0.69 * 60000, st\n")
    env = dict(os.environ, STEMROOT_DIST_GIANT="0")
    r = subprocess.run([sys.executable, "-c", code], cwd=ROOT, env=env, capture_output=True, text=True, timeout=600)
    assert r.returncode == 0, r.stderr[-3000:]


def test_nccl_single_rank(sr):
    import torch
    sp = G.spec("C1")
    kid, t, _ = G.generate_np(sp)
    try:
        uid = sr.nccl_unique_id()
    except sr.StemError as e:
        pytest.skip(f"NCCL unavailable: {e}")
    comm = sr.Comm.nccl(uid, 0, 1, 0)
    ctx = sr.Context(0)
    dk = torch.from_numpy(kid.view(np.int32)).cuda()
    dt = torch.from_numpy(t.view(np.int32)).cuda()
    got = ctx.plan_dist(comm, dk, dt, sp.n_kernels, 0, z=Z95, seed=2)
    ref = O.plan(kid, t, sp.n_kernels, z=Z95, seed=2)
    assert_plans_equal(got, ref)
    ctx.close()
    comm.close()


@pytest.mark.parametrize("world", [2, 3])
def test_packed_sort_candidate_rows_dist(sr, monkeypatch, world):
    """packed sort key with a forced small packing (many candidate rows per
    sample) under the multi-GPU row mapping (local index -> global row)"""
    monkeypatch.setenv("STEMROOT_PACK_BITS", "9")
    rng = np.random.default_rng(world)
    kid = rng.integers(0, 5, 30_011).astype(np.uint32)
    t = (rng.integers(0, 4, 30_011) * 300 + 1000 + kid * 7).astype(np.uint32)
    ref = O.plan(kid, t, 5, eps=0.002, z=Z95, seed=8)
    got = _dist_plan(sr, kid, t, 5, world, eps=0.002, z=Z95, seed=8)
    assert_plans_equal(got, ref)


def test_loopback_lloyd_split(sr):
    """the Lloyd split variant (opts.split = 1) is independent of the rank count too"""
    sp = G.spec("C2", n=120_000)
    kid, t, _ = G.generate_np(sp)
    ref = O.plan(kid, t, sp.n_kernels, eps=0.04, z=Z95, seed=6, split=1)
    got = _dist_plan(sr, kid, t, sp.n_kernels, 3, eps=0.04, z=Z95, seed=6, split=1)
    assert_plans_equal(got, ref)


def test_loopback_kmeans_split(sr):
    """the k-means split (split = 3, R29) decides on each cluster's own rows: independent of the rank count"""
    rng = np.random.default_rng(31)
    kid = rng.integers(0, 9, 30_000).astype(np.uint32)
    t = (rng.integers(0, 80, 30_000) * 53 + 2000 + kid * 9000).astype(np.uint32)
    ref = O.plan(kid, t, 9, eps=0.02, z=Z95, seed=2, split=3, kmeans_k=4)
    for world in (2, 3):
        got = _dist_plan(sr, kid, t, 9, world, eps=0.02, z=Z95, seed=2, split=3, kmeans_k=4)
        assert_plans_equal(got, ref)


def test_loopback_kmpp_split(sr):
    """the k-means++ split variant (opts.split = 2, R27) draws its seeds from the
    cluster's values only, so the plan is independent of the rank count"""
    sp = G.spec("C2", n=120_000)
    kid, t, _ = G.generate_np(sp)
    ref = O.plan(kid, t, sp.n_kernels, eps=0.04, z=Z95, seed=77, split=2)
    for world in (2, 3):
        got = _dist_plan(sr, kid, t, sp.n_kernels, world, eps=0.04, z=Z95, seed=77, split=2)
        assert_plans_equal(got, ref)


def test_loopback_rank_local_error_is_agreed(sr):
    """a failure on one rank only (here rank 1 passes n_kernels = 0,
    STEM_E_RANGE) makes every rank return that status, instead of the healthy
    ranks blocking in a collective."""
    import torch
    world = 3
    rng = np.random.default_rng(3)
    kid = rng.integers(0, 4, 9000).astype(np.uint32)
    t = rng.integers(100, 5000, 9000).astype(np.uint32)
    comms = sr.Comm.loopback(world, 0)
    ctxs = [sr.Context(0) for _ in range(world)]
    streams = [torch.cuda.Stream() for _ in range(world)]
    res = [None] * world

    def run(r):
        a, b = 3000 * r, 3000 * (r + 1)
        dk = torch.from_numpy(kid[a:b].view(np.int32)).cuda()
        dt = torch.from_numpy(t[a:b].view(np.int32)).cuda()
        try:
            ctxs[r].plan_dist(comms[r], dk, dt, 0 if r == 1 else 4, a, z=Z95, stream=streams[r].cuda_stream)
            res[r] = 0
        except sr.StemError as e:
            res[r] = e.status
    th = [threading.Thread(target=run, args=(r,)) for r in range(world)]
    for x in th:
        x.start()
    for x in th:
        x.join(timeout=120)
    assert not any(x.is_alive() for x in th), "a rank hung"
    assert res == [sr.STEM_E_RANGE] * world, res
    for c in ctxs:
        c.close()
    for c in comms:
        c.close()


def test_loopback_missing_peer_times_out(tmp_path):
    """A peer that never joins: the others give up after STEMROOT_COMM_TIMEOUT_S
    with STEM_E_NCCL (the NCCL communicator polls ncclCommGetAsyncError with the
    same timeout) instead of hanging."""
    import subprocess
    import sys
    prog = tmp_path / "miss.py"
    prog.write_text(
        "import sys, threading, numpy as np, torch\n"
        f"sys.path.insert(0, {ROOT!r})\n"
        "import paper_conf_micro_chungnkk25_b200 as sr\n"
        "comms = sr.Comm.loopback(2, 0)\n"
        "ctx = sr.Context(0)\n"
        "k = torch.zeros(100, dtype=torch.int32, device='cuda'); t = torch.arange(100, dtype=torch.int32, device='cuda')\n"
        "try:\n"
        "    ctx.plan_dist(comms[0], k, t, 1, 0)\n"
        "    print('NO-ERROR')\n"
        "except sr.StemError as e:\n"
        "    print('STATUS', e.status)\n")
    env = dict(os.environ, STEMROOT_COMM_TIMEOUT_S="3")
    out = subprocess.run([sys.executable, str(prog)], env=env, capture_output=True, text=True, timeout=300)
    assert "STATUS -5" in out.stdout, out.stdout + out.stderr


def test_fused_exchange_and_send_recv_paths_agree(tmp_path):
    """The kernel-id exchange stores rows straight into the owners' receive
    windows (stats.fused_exchange = 1; loopback windows are the other ranks'
    device buffers, NCCL ones CUDA-IPC peer memory); STEMROOT_DIST_P2P=0 keeps
    the grouped send/recv path.  Both give the single-trace oracle plan."""
    import subprocess
    import sys
    prog = tmp_path / "fx.py"
    prog.write_text(
        "import sys, threading, numpy as np, torch\n"
        f"sys.path.insert(0, {ROOT!r}); sys.path.insert(0, {os.path.join(ROOT, 'tests')!r})\n"
        "import paper_conf_micro_chungnkk25_b200 as sr, oracle as O, tracegen as G\n"
        "from parity_util import Z95, assert_plans_equal\n"
        "sp = G.spec('C2', n=90_000); kid, t, _ = G.generate_np(sp); W = 3\n"
        "cuts = [len(kid) * r // W for r in range(W + 1)]\n"
        "comms = sr.Comm.loopback(W, 0); ctxs = [sr.Context(0) for _ in range(W)]\n"
        "out = [None] * W; fx = [None] * W\n"
        "def run(r):\n"
        "    a, b = cuts[r], cuts[r + 1]\n"
        "    dk = torch.from_numpy(kid[a:b].view(np.int32)).cuda(); dt = torch.from_numpy(t[a:b].view(np.int32)).cuda()\n"
        "    out[r] = ctxs[r].plan_dist(comms[r], dk, dt, sp.n_kernels, a, z=Z95, seed=3, stream=torch.cuda.Stream().cuda_stream)\n"
        "    fx[r] = ctxs[r].stats()['fused_exchange']\n"
        "th = [threading.Thread(target=run, args=(r,)) for r in range(W)]\n"
        "[x.start() for x in th]; [x.join() for x in th]\n"
        "assert_plans_equal(out[0], O.plan(kid, t, sp.n_kernels, z=Z95, seed=3))\n"
        "print('FUSED', fx)\n")
    for env, want in (({}, "FUSED [1, 1, 1]"), ({"STEMROOT_DIST_P2P": "0"}, "FUSED [0, 0, 0]")):
        out = subprocess.run([sys.executable, str(prog)], env=dict(os.environ, **env), capture_output=True, text=True,
                             timeout=600)
        assert want in out.stdout, out.stdout + out.stderr[-3000:]
