"""Pins for the oracle (oracle/stemroot_oracle.c) against things other than itself:
hand-computed vectors from PAPER.md's formulas (tests/golden/*.json, each with
its citation), closed forms, brute force on tiny inputs, library routines
(math.fsum, Python's int->float, mpmath/scipy quantiles, Random123 KAT),
invariants (Theorem 3.1, partition, census exactness) and Monte-Carlo
coverage of the stated bound.  No GPU needed."""
import itertools
import math
import random
from fractions import Fraction

import numpy as np
import pytest

import oracle as O

Z95 = 1.959963984540054  # scipy.stats.norm.ppf(0.975)


# ----------------------------------------------------------------- Eq. 3 (P1)
def test_eq3_hand_vectors(golden):
    g = golden("eq3_hand.json")
    for c in g["cases"]:
        t = c["t"]
        n, S, Q = len(t), sum(t), sum(x * x for x in t)
        assert O.eq3_m(n, S, Q, c["eps"], c["z"]) == c["m"], c


def test_eq3_matches_textbook_form():
    # Eq. 3 is the textbook CLT sample size ceil((z*CoV/eps)^2) with population sigma.
    rng = random.Random(7)
    agree = 0
    for _ in range(500):
        t = [rng.randint(1, 10_000) for _ in range(rng.randint(2, 40))]
        n, S, Q = len(t), sum(t), sum(x * x for x in t)
        mu = S / n
        sigma = math.sqrt(sum((x - mu) ** 2 for x in t) / n)
        x = (1.96 * sigma / (mu * 0.05)) ** 2
        m = O.eq3_m(n, S, Q, 0.05, 1.96)
        assert abs(m - max(1, math.ceil(x))) <= 1
        agree += m == max(1, math.ceil(x))
    assert agree >= 495


# ----------------------------------------------------------------- Eq. 6 (P2, P2b, P2c, P3)
def test_eq6_hand_vectors(golden):
    g = golden("eq6_hand.json")
    for c in g["cases"]:
        m = O.eq6_m(c["mu"], c["V"], c["T"], c["eps"], c["z"])
        assert list(m) == c["m"], c
        w = c["eps"] * c["T"] / c["z"]
        assert w * w == pytest.approx(c["c"], rel=1e-15)
        if "tau_joint" in c:
            tau = sum(mi * a for mi, a in zip(m, c["mu"]))
            assert tau == c["tau_joint"] <= c["tau_indep"]


def test_eq6_printed_numerator_violates_bound():
    # Reading R1: with the printed sqrt(sum a_j b_j) numerator the constraint Eq. 5 fails.
    a, b, T = [2.0, 12.0], [6.0, 6.0], 42.0
    c = (0.05 * T / 1.96) ** 2
    printed = [math.sqrt(sum(x * y for x, y in zip(a, b))) / c * math.sqrt(bi / ai) for ai, bi in zip(a, b)]
    derived = [sum(math.sqrt(x * y) for x, y in zip(a, b)) / c * math.sqrt(bi / ai) for ai, bi in zip(a, b)]
    assert sum(bi / mi for bi, mi in zip(b, printed)) > c * 1.3
    assert sum(bi / mi for bi, mi in zip(b, derived)) == pytest.approx(c, rel=1e-12)
    m = O.eq6_m(a, b, T, 0.05, 1.96)
    assert sum(bi / mi for bi, mi in zip(b, m)) <= c


def test_eq6_single_cluster_reduces_to_eq3():
    # P2b: for k = 1, (sqrt(ab)/c)*sqrt(b/a) = b/c = (z sigma/(eps mu))^2 -- Eq. 6 == Eq. 3.
    rng = random.Random(11)
    same = 0
    for _ in range(400):
        t = [rng.randint(1, 5000) for _ in range(rng.randint(2, 30))]
        n, S, Q = len(t), sum(t), sum(x * x for x in t)
        V = n * Q - S * S
        if V == 0:
            continue
        m6 = O.eq6_m([S / n], [float(V)], S, 0.05, 1.96)[0]
        m3 = O.eq3_m(n, S, Q, 0.05, 1.96)
        assert abs(m6 - m3) <= 1
        same += m6 == m3
    assert same >= 390


def test_eq6_kkt_conditions():
    # App. 9.1: stationarity m*^2 a_i / b_i equal across i, Eq. 5 tight at m*,
    # and the ceiled solution stays feasible.
    rng = np.random.default_rng(3)
    for _ in range(200):
        k = int(rng.integers(2, 8))
        a = rng.uniform(1, 1000, k)
        b = rng.uniform(1, 1e6, k) * a
        T = float(a.sum() * rng.uniform(5, 50))
        eps, z = 0.05, 1.96
        c = (eps * T / z) ** 2
        mstar = np.sqrt(a * b).sum() / c * np.sqrt(b / a)
        lam = mstar ** 2 * a / b
        assert np.allclose(lam, lam[0], rtol=1e-12)
        assert (b / mstar).sum() == pytest.approx(c, rel=1e-12)
        m = O.eq6_m(a, b, T, eps, z)
        assert np.all(m == np.maximum(1, np.ceil(mstar)))
        assert (b / m).sum() <= c * (1 + 1e-12)


def test_eq6_integer_brute_force():
    # P2c: tau* <= tau_int_opt <= tau(ceil m*) < tau* + sum a_i ("minor sub-optimality").
    rng = random.Random(5)
    for _ in range(60):
        k = rng.randint(1, 3)
        a = [rng.randint(1, 20) for _ in range(k)]
        b = [rng.randint(1, 400) for _ in range(k)]
        T = sum(a) * rng.randint(2, 6)
        eps, z = 0.25, 1.0
        c = (eps * T / z) ** 2
        mstar = [sum(math.sqrt(x * y) for x, y in zip(a, b)) / c * math.sqrt(bi / ai) for ai, bi in zip(a, b)]
        tau_star = sum(m * x for m, x in zip(mstar, a))
        m = O.eq6_m(a, b, T, eps, z)
        tau_ceil = sum(mi * x for mi, x in zip(m, a))
        assert sum(bi / mi for bi, mi in zip(b, m)) <= c * (1 + 1e-12)
        hi = int(max(m)) + 2
        best = min(sum(mi * x for mi, x in zip(ms, a))
                   for ms in itertools.product(range(1, hi + 1), repeat=k)
                   if sum(Fraction(bi) / mi for bi, mi in zip(b, ms)) <= Fraction(c))
        assert tau_star - 1e-9 <= best <= tau_ceil + 1e-9
        assert tau_ceil < tau_star + sum(a) + 1e-9 or max(mstar) < 1


# ----------------------------------------------------------------- 2-means split (P4, P4b)
def _sse(vals):
    if not vals:
        return Fraction(0)
    mu = Fraction(sum(vals), len(vals))
    return sum((Fraction(v) - mu) ** 2 for v in vals)


def test_split_is_optimal_two_means_brute_force():
    rng = random.Random(17)
    for _ in range(600):
        n = rng.randint(2, 10)
        t = sorted(rng.choice([rng.randint(0, 6), rng.randint(0, 60)]) for _ in range(n))
        k = O.best_cut(t)
        if t[0] == t[-1]:
            assert k == 0
            continue
        assert 1 <= k < n and t[k - 1] < t[k]
        best = min(_sse([t[i] for i in range(n) if mask >> i & 1]) + _sse([t[i] for i in range(n) if not mask >> i & 1])
                   for mask in range(1, 2 ** n - 1))
        assert _sse(t[:k]) + _sse(t[k:]) == best
        # smallest k among the optimal distinct-value cuts
        first = min(j for j in range(1, n) if t[j - 1] < t[j] and _sse(t[:j]) + _sse(t[j:]) == best)
        assert k == first


def test_lloyd_variant_fixed_point_and_bounds():
    """split=1 (reading R26): Lloyd's k-means with k = 2 from the (min, max)
    centroids.  Pinned by what Lloyd's algorithm guarantees,
    not by retyping it: the returned cut is a fixed point of the assignment
    step (every value is on the side of its nearer centroid, ties to the left),
    it never separates equal values, its SSE is no better than the brute-force
    optimum and equals it on two well-separated groups, and on some inputs the
    local optimum it stops at is strictly worse than the global one (so the
    option really is a different split rule from the default)."""
    rng = random.Random(23)
    worse = 0
    for _ in range(800):
        n = rng.randint(2, 11)
        t = sorted(rng.choice([rng.randint(0, 6), rng.randint(0, 60), rng.randint(0, 600)]) for _ in range(n))
        k, iters = O.lloyd_cut(t)
        if t[0] == t[-1]:
            assert k == 0
            continue
        assert 1 <= k < n and t[k - 1] < t[k] and iters >= 1
        c1, c2 = Fraction(sum(t[:k]), k), Fraction(sum(t[k:]), n - k)
        assert all(2 * x <= c1 + c2 for x in t[:k]) and all(2 * x > c1 + c2 for x in t[k:])
        best = min(_sse(t[:j]) + _sse(t[j:]) for j in range(1, n))   # contiguous cuts suffice (1-D)
        mine = _sse(t[:k]) + _sse(t[k:])
        assert mine >= best
        worse += mine > best
    assert worse > 0
    for _ in range(50):   # two well-separated groups: the global optimum
        a = [rng.randint(0, 50) for _ in range(rng.randint(1, 8))]
        b = [10_000 + rng.randint(0, 50) for _ in range(rng.randint(1, 8))]
        t = sorted(a + b)
        assert O.lloyd_cut(t)[0] == len(a) == O.best_cut(t)


def test_kmpp_seeds_follow_d2_weighting():
    """split=2 (reading R27): the k-means++ seeds.  Pinned by the definition of
    D^2 seeding (Arthur & Vassilvitskii): c1 is a uniform row, and given c1 the
    second seed is row j with probability (t_j - c1)^2 / sum_i (t_i - c1)^2.
    Over 24 000 seeds the joint frequency of (c1, c2) values must match those
    exact probabilities (each cell within 5 binomial standard deviations) and
    a zero-probability pair (c2 == c1) must never occur."""
    t = [3, 3, 5, 9, 9, 9, 14, 20]
    n = len(t)
    vals = sorted(set(t))
    cnt = {v: t.count(v) for v in vals}
    prob = {}
    for a in vals:
        W = sum((x - a) ** 2 for x in t)
        for b in vals:
            prob[(a, b)] = Fraction(cnt[a], n) * Fraction(cnt[b] * (b - a) ** 2, W)
    R = 24_000
    seen = {}
    for s in range(R):
        k, c1, c2, it = O.kmpp_cut(t, 0x9E3779B97F4A7C15 * (s + 1))
        assert c1 in cnt and c2 in cnt and c1 != c2 and 1 <= k < n and t[k - 1] < t[k] and it >= 1
        seen[(c1, c2)] = seen.get((c1, c2), 0) + 1
    for key, p in prob.items():
        e = float(p) * R
        sd = math.sqrt(max(e * (1 - float(p)), 1e-9))
        assert abs(seen.get(key, 0) - e) <= 5 * sd + 1e-9, (key, seen.get(key, 0), e)


def test_kmpp_variant_fixed_point_and_bounds():
    """split=2 (R27): whatever the seeds, the result is a Lloyd fixed point on
    the exact fractional centroids (ties to the left), never separates equal
    values, never beats the brute-force optimum, finds it on two well-separated
    groups, is a pure function of (values, seed), and different seeds reach
    different local optima on some inputs (the seeding is really random)."""
    rng = random.Random(31)
    differ = 0
    for case in range(600):
        n = rng.randint(2, 11)
        t = sorted(rng.choice([rng.randint(0, 6), rng.randint(0, 60), rng.randint(0, 600)]) for _ in range(n))
        k, c1, c2, it = O.kmpp_cut(t, case)
        assert O.kmpp_cut(t, case) == (k, c1, c2, it)
        if t[0] == t[-1]:
            assert k == 0
            continue
        assert 1 <= k < n and t[k - 1] < t[k] and it >= 1 and c1 != c2 and c1 in t and c2 in t
        m1, m2 = Fraction(sum(t[:k]), k), Fraction(sum(t[k:]), n - k)
        assert all(2 * x <= m1 + m2 for x in t[:k]) and all(2 * x > m1 + m2 for x in t[k:])
        best = min(_sse(t[:j]) + _sse(t[j:]) for j in range(1, n))
        assert _sse(t[:k]) + _sse(t[k:]) >= best
        differ += len({O.kmpp_cut(t, s)[0] for s in range(40)}) > 1
    assert differ > 0
    for _ in range(50):
        a = [rng.randint(0, 50) for _ in range(rng.randint(1, 8))]
        b = [10_000 + rng.randint(0, 50) for _ in range(rng.randint(1, 8))]
        tt = sorted(a + b)
        assert O.kmpp_cut(tt, rng.getrandbits(64))[0] == len(a) == O.best_cut(tt)


def test_kmpp_plan_option():
    """or_opts.split = 2 builds a valid partition, depends on the seed only
    through the split, and the oracle rejects split = 4"""
    rng = np.random.default_rng(4)
    kid = rng.integers(0, 5, 4000).astype(np.uint32)
    t = (rng.lognormal(8, 0.6, 4000) + 1000 * (rng.random(4000) < 0.3)).astype(np.uint32)
    p = O.plan(kid, t, 5, eps=0.03, z=Z95, seed=1, split=2)
    assert int(np.sum(p["n"])) == 4000
    assert O.plan(kid, t, 5, eps=0.03, z=Z95, seed=1, split=2)["n"].tolist() == p["n"].tolist()
    with pytest.raises(Exception):
        O.plan(kid, t, 5, eps=0.03, z=Z95, seed=1, split=4)


def test_split_exact_tie(golden):
    for c in golden("split_tie.json")["cases"]:
        t = [c["s"] * x for x in c["base"]]
        assert O.best_cut(t) == c["cut"]


# ----------------------------------------------------------------- ROOT trees (P5, P5b)
def test_root_worked_trees(golden):
    g = golden("root_trees.json")
    for tr in g["trees"]:
        split, to, tn, cut = O.root_decide(tr["t"], tr["eps"], tr["z"])
        r = tr["root"]
        assert (split, to, tn, cut) == (r["split"], r["tau_old"], r["tau_new"], r["cut"])
        for seed in (0, 1, 12345):
            p = O.plan([0] * len(tr["t"]), tr["t"], 1, eps=tr["eps"], z=tr["z"], seed=seed)
            assert [[int(a), int(b)] for a, b in zip(p["lo_ns"], p["hi_ns"])] == tr["leaves_lo_hi"]
            assert list(p["m"]) == tr["m"]
            assert p["est_total_ns"] == tr["est"] and p["bound"] == tr["bound"]
    for st in g["subtrees"]:
        split, to, tn, cut = O.root_decide(st["t"], st["eps"], st["z"])
        assert (split, to, tn, cut) == (st["split"], st["tau_old"], st["tau_new"], st["cut"])


def test_stem_only_two_kernels(golden):
    c = golden("eq6_hand.json")["cases"][1]
    p = O.plan([0, 0, 0, 0, 1, 1, 1, 1], [10, 20, 30, 40, 100, 100, 100, 300], 2, eps=0.05, z=1.96, root=0)
    assert list(p["m"]) == c["m"]
    assert p["ssum"] == pytest.approx(c["ssum"], rel=1e-15)
    # bound = z sqrt(sum V/m)/T (Eq. 5 at the realised m), below eps
    b = 1.96 * math.sqrt(2000 / 126 + 120000 / 397) / 700
    assert p["bound"] == pytest.approx(b, rel=1e-14) and p["bound"] <= 0.05


# ----------------------------------------------------------------- primitives
def test_philox_kat(golden):
    for c in golden("philox_kat.json")["cases"]:
        out = O.philox4x32_10([int(x, 16) for x in c["ctr"]], [int(x, 16) for x in c["key"]])
        assert out == [int(x, 16) for x in c["out"]]


def test_z_from_conf_against_mpmath_and_scipy():
    import mpmath
    from scipy.stats import norm
    mpmath.mp.dps = 40
    for conf in (0.5, 0.8, 0.9, 0.95, 0.975, 0.99, 0.999, 0.999999, 1 - 1e-12):
        p = 1 - (1 - conf) / 2
        ref = float(mpmath.sqrt(2) * mpmath.erfinv(2 * mpmath.mpf(p) - 1))
        z = O.z_from_conf(conf)
        assert abs(z - ref) <= 4 * math.ulp(ref), (conf, z, ref)
        assert z == pytest.approx(norm.ppf(p), rel=1e-14)
    assert math.isnan(O.z_from_conf(1.0)) and math.isnan(O.z_from_conf(0.0))


def test_u128_to_double_rounding():
    rng = random.Random(23)
    cases = [0, 1, 2 ** 53 + 1, 2 ** 64 - 1, 2 ** 64, 2 ** 64 + 2 ** 11, 2 ** 128 - 1,
             (2 ** 53 + 1) << 70, ((2 ** 53 + 1) << 70) + 1, (2 ** 54 + 2) << 60, ((2 ** 54 + 2) << 60) + 1]
    for _ in range(20000):
        bits = rng.randint(1, 128)
        v = rng.getrandbits(bits)
        if rng.random() < 0.3:  # near-tie patterns: 1 bit beyond the mantissa, maybe sticky
            top = max(bits - 54, 0)
            v = (v >> top << top) | (1 << max(top - 1, 0)) if top else v
        cases.append(v)
    for v in cases:
        assert O.u128_to_double(v) == float(v), v  # Python int->float is correctly rounded


def test_exact_sum_against_fsum():
    rng = np.random.default_rng(29)
    for _ in range(50):
        n = int(rng.integers(0, 3000))
        x = np.exp(rng.uniform(-11, 55, n))  # the KKT terms live in [2^-16, 2^80)
        x[rng.random(n) < 0.05] = 0.0
        assert O.exact_sum(x) == math.fsum(x)
    # cancellation-free but order-sensitive case: naive summation differs, exact does not
    x = np.array([2.0 ** 80] + [1.0] * 5000 + [2.0 ** -16] * 7)
    assert O.exact_sum(x) == math.fsum(x) == O.exact_sum(x[::-1])


# ----------------------------------------------------------------- invariants (P6, P7, P8)
def _random_trace(rng, n, k, max_t=2 ** 20):
    kid = rng.integers(0, k, n).astype(np.uint32)
    centers = rng.integers(1000, max_t, (k, 3))
    peak = rng.integers(0, 3, n)
    t = (centers[kid, peak] * rng.lognormal(0, 0.05, n)).astype(np.uint64)
    return kid, np.minimum(t, 2 ** 32 - 1).astype(np.uint32)


@pytest.mark.parametrize("scope", [0, 1, 2])
@pytest.mark.parametrize("eps", [0.01, 0.05, 0.2])
def test_plan_invariants(scope, eps):
    rng = np.random.default_rng(int(eps * 1000) + scope)
    kid, t = _random_trace(rng, 4000, 7)
    p = O.plan(kid, t, 7, eps=eps, z=Z95, seed=3, scope=scope)
    L = len(p["n"])
    # partition: leaves cover each group, sum n = N, no time value split across two leaves
    assert int(p["n"].sum()) == len(t)
    assert p["true_total_ns"] == int(t.astype(np.uint64).sum())
    for k in range(7):
        idx = np.nonzero(p["kernel_id"] == k)[0]
        sel = np.sort(t[kid == k])
        assert list(p["ordinal"][idx]) == list(range(len(idx)))
        assert np.all(p["hi_ns"][idx][:-1] < p["lo_ns"][idx][1:])
        assert p["lo_ns"][idx][0] == sel[0] and p["hi_ns"][idx][-1] == sel[-1]
        for i in idx:
            mem = sel[(sel >= p["lo_ns"][i]) & (sel <= p["hi_ns"][i])]
            assert len(mem) == p["n"][i] and int(mem.astype(np.uint64).sum()) == p["sum_ns"][i]
    assert np.all(np.diff(p["kernel_id"].astype(np.int64)) >= 0)
    # bound: global scope obeys Eq. 5; per-kernel / per-leaf obey it by Theorem 3.1
    assert p["bound"] <= eps
    assert np.all(p["m"] >= 1)
    # samples: ordered by cluster, each row belongs to its cluster, weight = n_i/m_i
    assert len(p["sample_row"]) == int(p["m"].sum())
    assert np.all(np.diff(p["sample_cluster"].astype(np.int64)) >= 0)
    c = p["sample_cluster"]
    rows = p["sample_row"]
    assert np.all(kid[rows] == p["kernel_id"][c])
    assert np.all((t[rows] >= p["lo_ns"][c]) & (t[rows] <= p["hi_ns"][c]))
    assert np.allclose(p["sample_weight"], p["n"][c].astype(float) / p["m"][c])
    assert L >= 7


def test_leaves_invariant_to_row_order():
    rng = np.random.default_rng(41)
    kid, t = _random_trace(rng, 3000, 5)
    a = O.plan(kid, t, 5)
    perm = rng.permutation(len(t))
    b = O.plan(kid[perm], t[perm], 5)
    for key in ("kernel_id", "ordinal", "lo_ns", "hi_ns", "n", "sum_ns", "m"):
        assert np.array_equal(a[key], b[key])


def test_census_is_exact():
    # P8: census_cap with a tiny eps takes every row once -> estimate == T exactly (north_star)
    rng = np.random.default_rng(43)
    kid, t = _random_trace(rng, 2000, 4)
    met = np.vstack([t.astype(float), np.ones(len(t))])
    p = O.plan(kid, t, 4, eps=1e-6, census_cap=1, root=0, metrics=met)
    assert p["census"].all()
    assert p["est_total_ns"] == float(p["true_total_ns"])
    assert sorted(p["sample_row"]) == list(range(len(t)))
    assert p["est_metric"][0] == pytest.approx(float(t.astype(np.float64).sum()), rel=1e-12)
    assert p["est_metric"][1] == pytest.approx(len(t), rel=1e-12)
    # with ROOT every leaf is either a census or constant (sigma = 0): still exact
    p = O.plan(kid, t, 4, eps=1e-6, census_cap=1, metrics=met)
    assert np.all((p["census"] == 1) | (p["lo_ns"] == p["hi_ns"]))
    assert p["est_total_ns"] == float(p["true_total_ns"])


def test_constant_and_singleton_kernels_are_exact():
    kid = np.array([0, 0, 0, 1, 2, 2], np.uint32)
    t = np.array([5, 5, 5, 9, 0, 0], np.uint32)
    p = O.plan(kid, t, 3)
    assert list(p["n"]) == [3, 1, 2] and list(p["m"]) == [1, 1, 1]
    assert p["est_total_ns"] == 24.0 and p["bound"] == 0.0


def test_error_codes():
    with pytest.raises(O.OracleError) as e:
        O.plan([0, 3], [1, 2], 3)
    assert e.value.status == O.OR_E_RANGE
    for eps in (0.0, 1.0, -1.0):
        with pytest.raises(O.OracleError) as e:
            O.plan([0], [1], 1, eps=eps)
        assert e.value.status == O.OR_E_INVAL


def test_literal_clamp_reading_differs_only_in_split_test():
    # R7: clamp_in_split=0 uses literal ceilings (m may be 0 when sigma = 0) inside Eq. 7/8.
    kid = np.zeros(20, np.uint32)
    t = np.array([100] * 10 + [200] * 10, np.uint32)
    for cl in (0, 1):
        p = O.plan(kid, t, 1, clamp_in_split=cl, z=1.96)
        assert list(p["n"]) == [10, 10] and list(p["m"]) == [1, 1]


# ----------------------------------------------------------------- statistics (P9)
def test_sample_positions_uniform():
    # With replacement, uniform over the cluster: chi-square on a big cluster.
    rng = np.random.default_rng(47)
    t = rng.integers(1, 1000, 64).astype(np.uint32)
    p = O.plan(np.zeros(64, np.uint32), t, 1, eps=0.002, root=0, seed=99)
    rows = p["sample_row"]
    assert len(rows) > 20000
    counts = np.bincount(rows, minlength=64)
    exp = len(rows) / 64
    chi2 = ((counts - exp) ** 2 / exp).sum()
    assert chi2 < 120  # 63 dof: p ~ 3e-5


@pytest.mark.slow
def test_monte_carlo_unbiased_and_coverage():
    rng = np.random.default_rng(53)
    kid, t = _random_trace(rng, 3000, 6)
    # STEM only: m_i > 1, the CLT regime the paper models (Eq. 4/5)
    R = 300
    errs, cover = [], 0
    for seed in range(R):
        p = O.plan(kid, t, 6, eps=0.02, root=0, seed=seed)
        T = p["true_total_ns"]
        e = (p["est_total_ns"] - T) / T
        errs.append(e)
        cover += abs(e) <= p["bound"]
    errs = np.array(errs)
    assert abs(errs.mean()) < 4 * errs.std() / math.sqrt(R)
    assert 0.89 <= cover / R <= 0.995


# ----------------------------------------------------------------- leaf statistics (R3)
def test_std_ns_population_hand_vectors(golden):
    """std_ns is the population sigma of the leaf (reading R3), pinned by
    hand vectors (tests/golden/std_hand.json), not by the oracle's own formula."""
    g = golden("std_hand.json")
    kid, t = [], []
    for k, kern in enumerate(g["kernels"]):
        kid += [k] * len(kern["t"])
        t += kern["t"]
    p = O.plan(kid, t, len(g["kernels"]), eps=0.05, z=1.96, root=0)
    for k, kern in enumerate(g["kernels"]):
        assert p["mean_ns"][k] == kern["mean_ns"]
        assert p["std_ns"][k] == pytest.approx(kern["std_ns"], rel=1e-15)
        assert abs(p["std_ns"][k] - kern["sample_std"]) > 1.0   # not the n-1 form


def test_std_ns_against_numpy_on_random_leaves():
    """Every leaf's (mean_ns, std_ns) equals numpy's mean / std(ddof=0) of the
    leaf's member times (numpy is independent of the oracle's integer moments)."""
    rng = np.random.default_rng(59)
    kid, t = _random_trace(rng, 5000, 6)
    p = O.plan(kid, t, 6, eps=0.02, z=Z95, seed=1)
    for i in range(len(p["n"])):
        mem = t[(kid == p["kernel_id"][i]) & (t >= p["lo_ns"][i]) & (t <= p["hi_ns"][i])].astype(np.float64)
        assert len(mem) == p["n"][i]
        assert p["mean_ns"][i] == pytest.approx(mem.mean(), rel=1e-13)
        assert p["std_ns"][i] == pytest.approx(mem.std(), rel=1e-9, abs=1e-9 * mem.mean())


# ----------------------------------------------------------------- metric estimator (R18)
def _estimator_cases():
    for scope in (0, 1, 2):
        for root in (0, 1):
            for seed in (0, 5, 0xDEADBEEF):
                yield scope, root, seed


def _hash_metric(rows):
    x = rows.astype(np.uint64) * np.uint64(0x9E3779B97F4A7C15)
    x ^= x >> np.uint64(29)
    return (x % np.uint64(1_000_003)).astype(np.float64) / 7.0


def test_metric_estimator_weighted_sum_invariants():
    """The metric estimate is the weighted sum sum_i (n_i/m_i) sum_j metric[row_ij]
    (P:L371 'weighted sum', P:L107 weights; reading R18), pinned outside census
    mode (m_i > 1, samples with replacement) by three facts that a plausible
    mistake breaks:
      * a constant-1 column estimates N exactly (up to rounding): a swapped
        weight m_i/n_i gives sum m_i^2/n_i instead;
      * a column equal to t estimates est_total_ns: gathering metric[sorted
        position] instead of metric[trace row] reads other rows' values;
      * a column f(row) (a hash of the trace row) equals sum_s w_s f(row_s)
        over the plan's own sample rows and weights."""
    rng = np.random.default_rng(61)
    kid, t = _random_trace(rng, 6000, 5)
    rows = np.arange(len(t))
    met = np.vstack([np.ones(len(t)), t.astype(np.float64), _hash_metric(rows)])
    multi = 0
    for scope, root, seed in _estimator_cases():
        p = O.plan(kid, t, 5, eps=0.01, z=Z95, seed=seed, scope=scope, root=root, metrics=met)
        assert not p["census"].any()
        multi += int((p["m"] > 1).sum())
        assert p["est_metric"][0] == pytest.approx(len(t), rel=1e-12)
        assert p["est_metric"][1] == pytest.approx(p["est_total_ns"], rel=1e-12)
        direct = float(np.sum(p["sample_weight"] * _hash_metric(p["sample_row"])))
        assert p["est_metric"][2] == pytest.approx(direct, rel=1e-12)
    assert multi > 100   # the pins run where weights differ from 1


# ----------------------------------------------------------------- Lloyd trajectory (R26)
def test_lloyd_hand_traced_trajectory(golden):
    """split = 1 (reading R26): hand-traced Lloyd iterations from the (min, max)
    centroids (tests/golden/lloyd_trace.json, every step written out).  The
    oracle's cut and number of centroid updates must match the trace; a
    different initialisation (e.g. the two smallest values, or k-means++)
    takes a different number of steps or stops elsewhere."""
    for c in golden("lloyd_trace.json")["cases"]:
        k, updates = O.lloyd_cut(c["t"])
        assert (k, updates) == (c["cut"], c["updates"])
        assert O.best_cut(c["t"]) == c["best_cut"]
        # the trace's first step starts from (min, max): pin the reading, not just the result
        assert c["steps"][0][:2] == [str(min(c["t"])), str(max(c["t"]))]


# ----------------------------------------------------------------- metric totals and bounds (R28)
def test_exact_sum_signed_against_fsum():
    rng = np.random.default_rng(67)
    for n in (0, 1, 7, 1000, 20000):
        x = rng.standard_normal(n) * 10.0 ** rng.integers(-30, 30, n)
        assert O.exact_sum_signed(x) == math.fsum(x)
    x = np.array([1e300, 1.0, -1e300, 2.0 ** -1000, -3.0])
    assert O.exact_sum_signed(x) == math.fsum(x)


def test_metric_bounds_invariants():
    """metric_bounds (reading R28: Eq. 5 with the metric in place of the time,
    P:L150-159), pinned by what holds whatever the implementation:
      * true_metric is the column's exact sum (math.fsum, correctly rounded);
      * a metric equal to t reproduces the time bound (the oracle computes the
        time variance from exact integer moments and the metric variance by a
        separate fp64 two-pass, so a dropped n_i, a sample variance or a
        missing mean subtraction shows up);
      * an affine metric a t + b has bound |a| bound T / |a T + b N| (a shift
        leaves the variance alone, a scale multiplies it by a^2);
      * a constant column has bound 0; the other outputs are unchanged."""
    rng = np.random.default_rng(71)
    kid, t = _random_trace(rng, 5000, 5)
    N = len(t)
    tf = t.astype(np.float64)
    met = np.vstack([tf, 3.0 * tf + 1e6, -0.5 * tf, np.full(N, 7.25), rng.random(N) - 0.3])
    for scope, root, seed in [(0, 1, 0), (0, 0, 3), (1, 1, 9), (2, 1, 4), (0, 1, 77)]:
        p = O.plan(kid, t, 5, eps=0.01, z=Z95, seed=seed, scope=scope, root=root, metrics=met, metric_bounds=1)
        q = O.plan(kid, t, 5, eps=0.01, z=Z95, seed=seed, scope=scope, root=root, metrics=met)
        assert q["true_metric"] is None and q["bound_metric"] is None
        assert np.array_equal(p["m"], q["m"]) and np.array_equal(p["est_metric"], q["est_metric"])
        for c in range(met.shape[0]):
            assert p["true_metric"][c] == math.fsum(met[c])
        T, b = p["true_total_ns"], p["bound"]
        assert b > 0
        assert p["bound_metric"][0] == pytest.approx(b, rel=1e-10)
        assert p["bound_metric"][1] == pytest.approx(3.0 * b * T / (3.0 * T + 1e6 * N), rel=1e-10)
        assert p["bound_metric"][2] == pytest.approx(b, rel=1e-10)
        assert p["bound_metric"][3] == 0.0
        assert p["bound_metric"][4] > 0


def test_metric_bounds_census_exact():
    """census leaves (every row once): each metric estimate equals its true total."""
    rng = np.random.default_rng(73)
    kid, t = _random_trace(rng, 1500, 3)
    met = np.vstack([rng.random(len(t)), t.astype(np.float64) ** 0.5])
    p = O.plan(kid, t, 3, eps=1e-6, census_cap=1, root=0, metrics=met, metric_bounds=1)
    assert p["census"].all()
    for c in range(2):
        assert p["est_metric"][c] == pytest.approx(p["true_metric"][c], rel=1e-12)


@pytest.mark.slow
def test_metric_bound_monte_carlo_coverage():
    """bound_c is a z-level confidence bound of the metric estimate's relative
    error (CLT over the leaves' with-replacement samples): over 300
    seeds in the m_i > 1 regime the realised error is inside it about 95 % of
    the time, and the estimate is unbiased."""
    rng = np.random.default_rng(79)
    kid, t = _random_trace(rng, 3000, 6)
    met = np.vstack([t.astype(np.float64) * rng.uniform(0.5, 1.5, len(t)), rng.gamma(2.0, 3.0, len(t))])
    R = 300
    cover = np.zeros(2)
    errs = [[], []]
    for seed in range(R):
        p = O.plan(kid, t, 6, eps=0.02, root=0, seed=seed, metrics=met, metric_bounds=1)
        for c in range(2):
            e = (p["est_metric"][c] - p["true_metric"][c]) / p["true_metric"][c]
            errs[c].append(e)
            cover[c] += abs(e) <= p["bound_metric"][c]
    for c in range(2):
        e = np.array(errs[c])
        assert abs(e.mean()) < 4 * e.std() / math.sqrt(R)
        assert 0.89 <= cover[c] / R <= 0.995, cover


# ----------------------------------------------------------------- exact k-means, k > 2 (R29)
def _set_partitions(items, k):
    """every partition of the list into exactly k nonempty blocks"""
    if k == 1:
        yield [items]
        return
    if len(items) < k:
        return
    first, rest = items[0], items[1:]
    for p in _set_partitions(rest, k - 1):   # first alone
        yield [[first]] + p
    for p in _set_partitions(rest, k):       # first joins a block
        for i in range(len(p)):
            yield p[:i] + [[first] + p[i]] + p[i + 1:]


def _groups_from_cuts(t, cuts):
    b = [0] + list(cuts) + [len(t)]
    return [t[b[i]:b[i + 1]] for i in range(len(b) - 1)]


def test_kmeans_hand_vectors(golden):
    g = golden("kmeans_hand.json")
    for c in g["cuts"]:
        assert O.kmeans_cuts(c["t"], c["k"]) == c["cuts"], c
    tr = g["tree"]
    p = O.plan([0] * len(tr["t"]), tr["t"], 1, eps=tr["eps"], z=tr["z"], split=3, kmeans_k=tr["k"])
    assert [[int(a), int(b)] for a, b in zip(p["lo_ns"], p["hi_ns"])] == tr["leaves_lo_hi"]


def test_kmeans_is_the_global_optimum_brute_force():
    """R29: the DP's partition has the least SSE among ALL partitions of the
    multiset into min(k, #distinct) nonempty groups (not only contiguous ones),
    is contiguous in sorted order and never separates equal values."""
    rng = random.Random(83)
    for _ in range(300):
        n = rng.randint(2, 8)
        t = sorted(rng.choice([rng.randint(0, 5), rng.randint(0, 40)]) for _ in range(n))
        if t[0] == t[-1]:
            continue
        k = rng.randint(2, 4)
        d = len(set(t))
        K = min(k, d)
        cuts = O.kmeans_cuts(t, k)
        assert len(cuts) == K - 1 and all(t[c - 1] < t[c] for c in cuts) and cuts == sorted(cuts)
        mine = sum(_sse(g) for g in _groups_from_cuts(t, cuts))
        best = min(sum(_sse(g) for g in p) for p in _set_partitions(list(t), K))
        assert mine == best, (t, k, cuts)


def test_kmeans_tie_rule_brute_force():
    """Among the optimal contiguous distinct-value partitions the DP returns the
    one with the smallest last cut, then the smallest cut before it (R29)."""
    rng = random.Random(89)
    ties = 0
    for _ in range(400):
        n = rng.randint(3, 10)
        t = sorted(rng.choice([rng.randint(0, 3) * 10, rng.randint(0, 6) * 10]) for _ in range(n))
        if t[0] == t[-1]:
            continue
        k = rng.randint(2, 4)
        valid = [i for i in range(1, n) if t[i - 1] < t[i]]
        K = min(k, len(valid) + 1)
        cands = []
        for cut in itertools.combinations(valid, K - 1):
            cands.append((sum(_sse(g) for g in _groups_from_cuts(t, cut)), tuple(reversed(cut)), list(cut)))
        best = min(c[0] for c in cands)
        opt = [c for c in cands if c[0] == best]
        ties += len(opt) > 1
        assert O.kmeans_cuts(t, k) == min(opt, key=lambda c: c[1])[2], (t, k)
    assert ties > 20


def test_kmeans_k2_is_the_exact_two_means(golden):
    """k = 2 reduces to the exact 2-means cut of R5 (same objective, same tie rule)"""
    rng = random.Random(97)
    for _ in range(1500):
        n = rng.randint(2, 30)
        t = sorted(rng.choice([rng.randint(0, 4), rng.randint(0, 100), rng.randint(0, 5000)]) for _ in range(n))
        if t[0] == t[-1]:
            continue
        assert O.kmeans_cuts(t, 2) == [O.best_cut(t)]
    for c in golden("split_tie.json")["cases"]:
        t = [c["s"] * x for x in c["base"]]
        assert O.kmeans_cuts(t, 2) == [c["cut"]]


def test_kmeans_plan_k2_equals_default_split():
    rng = np.random.default_rng(101)
    kid, t = _random_trace(rng, 3000, 5)
    a = O.plan(kid, t, 5, eps=0.02, z=Z95, seed=3)
    b = O.plan(kid, t, 5, eps=0.02, z=Z95, seed=3, split=3, kmeans_k=2)
    for key in ("kernel_id", "ordinal", "lo_ns", "hi_ns", "n", "sum_ns", "m", "sample_row"):
        assert np.array_equal(a[key], b[key]), key
    assert a["est_total_ns"] == b["est_total_ns"] and a["bound"] == b["bound"]


@pytest.mark.parametrize("k", [3, 4, 8])
def test_kmeans_plan_invariants(k):
    rng = np.random.default_rng(103 + k)
    kid = rng.integers(0, 4, 2500).astype(np.uint32)
    t = (rng.integers(1, 60, 2500) * 37 + kid * 1000).astype(np.uint32)   # few distinct values per kernel
    p = O.plan(kid, t, 4, eps=0.02, z=Z95, seed=5, split=3, kmeans_k=k)
    assert int(p["n"].sum()) == len(t) and p["true_total_ns"] == int(t.astype(np.uint64).sum())
    for kk in range(4):
        idx = np.nonzero(p["kernel_id"] == kk)[0]
        assert np.all(p["hi_ns"][idx][:-1] < p["lo_ns"][idx][1:])
    assert p["bound"] <= 0.02 and np.all(p["m"] >= 1)
    with pytest.raises(O.OracleError):
        O.plan(kid, t, 4, split=3, kmeans_k=1)
