"""The nearest-centre lemma the GPU split relies on (DESIGN.md §5c,
root.cu nc_split_kernel), checked by brute force with exact rationals, no GPU.

For sorted integer times, every maximiser k* of D_k^2 / (k (n - k)) over the
valid cuts (t[k-1] < t[k]) -- the exact 2-means optimum the oracle computes
 -- satisfies t[k*-1] <= m(k*) <= t[k*] with
m(k) = (mu_L(k) + mu_R(k)) / 2, and m is non-decreasing in k.  The descent
prunes a range of cuts [a, b] when m(b) < t[a-1] or m(a) > t[b]; these tests
pin both facts (and the integer form of the comparison) on random, tie-heavy
and adversarial multimodal inputs, so a wrong sign or index in the lemma would
show here before any kernel runs."""
from fractions import Fraction

import numpy as np
import pytest


def _scores(t):
    n = len(t)
    S = int(sum(t))
    SL = 0
    out = []
    for k in range(1, n):
        SL += int(t[k - 1])
        D = n * SL - S * k
        out.append((k, SL, Fraction(D * D, k * (n - k))))
    return S, out


def _m(S, SL, k, n):
    return (Fraction(SL, k) + Fraction(S - SL, n - k)) / 2


def _cases():
    rng = np.random.default_rng(2024)
    for i in range(300):
        n = int(rng.integers(2, 90))
        kind = i % 5
        if kind == 0:
            t = rng.integers(0, 50, n)                     # many ties
        elif kind == 1:
            t = rng.integers(0, 2 ** 32, n, dtype=np.uint64)   # full range
        elif kind == 2:
            c = rng.integers(100, 10_000, 4)
            t = c[rng.integers(0, 4, n)] + rng.integers(0, 30, n)   # multimodal
        elif kind == 3:
            t = np.r_[np.full(n // 2 + 1, 7), rng.integers(0, 1000, n // 2 + 1)]   # a dominant run
        else:
            t = (rng.lognormal(8, 1.2, n)).astype(np.int64)   # heavy tail
        yield np.sort(np.asarray(t, dtype=object))


@pytest.mark.parametrize("chunk", list(range(6)))
def test_optimal_cut_satisfies_nearest_centre_condition(chunk):
    cases = list(_cases())[chunk * 50:(chunk + 1) * 50]
    for t in cases:
        n = len(t)
        S, sc = _scores(t)
        valid = [(k, SL, f) for k, SL, f in sc if t[k - 1] < t[k]]
        if not valid:
            continue
        best = max(f for _, _, f in valid)
        for k, SL, f in valid:
            m = _m(S, SL, k, n)
            if f == best:   # every maximiser (so every tie) satisfies the condition
                assert t[k - 1] <= m <= t[k], (list(t), k)
            # integer form used on the GPU: m(k) >= v  <=>  SL (n-k) + (S-SL) k >= 2 v k (n-k)
            for v in (int(t[k - 1]), int(t[k])):
                F = SL * (n - k) + (S - SL) * k
                assert (m >= v) == (F >= 2 * v * k * (n - k))
                assert (m <= v) == (F <= 2 * v * k * (n - k))


def test_midpoint_is_monotone_and_range_pruning_is_safe():
    for t in list(_cases())[:120]:
        n = len(t)
        S, sc = _scores(t)
        ms = [_m(S, SL, k, n) for k, SL, _ in sc]
        assert all(a <= b for a, b in zip(ms, ms[1:]))
        valid = [(k, f) for k, _, f in sc if t[k - 1] < t[k]]
        if not valid:
            continue
        best = max(f for _, f in valid)
        arg = [k for k, f in valid if f == best]
        # every range [a, b] holding a maximiser survives the descent's test
        for a in range(1, n):
            for b in range(a, n):
                if not any(a <= k <= b for k in arg):
                    continue
                assert t[a - 1] < t[b]
                assert ms[b - 1] >= t[a - 1] and ms[a - 1] <= t[b]


def test_kmeans_between_group_form():
    """The k-means option's fp64 filter (kmeans.cu km_between) evaluates the DP in
    between-group form: for prefix sums S, counts n over sorted distinct values,
    S(0,a)^2/n(0,a) + S(a,b)^2/n(a,b) - S(0,b)^2/n(0,b)
        = (n(a,b) S(0,a) - n(0,a) S(a,b))^2 / (n(0,a) n(a,b) n(0,b)),
    so G[j][b] = F[j][b] - S(0,b)^2/n(0,b) obeys G[j][b] = max_a G[j-1][a] + T(a,b)
    with the same argmax as the F recurrence.  Checked with exact rationals."""
    rng = np.random.default_rng(77)
    for _ in range(40):
        d = int(rng.integers(3, 14))
        cnt = rng.integers(1, 50, d)
        val = np.cumsum(rng.integers(1, 10_000, d))          # distinct sorted values
        n = np.r_[0, np.cumsum(cnt)].astype(object)
        S = np.r_[0, np.cumsum(cnt * val)].astype(object)

        def T(a, b):
            na, nab, nb = n[a], n[b] - n[a], n[b]
            Sa, Sab = S[a], S[b] - S[a]
            return Fraction((nab * Sa - na * Sab) ** 2, na * nab * nb)

        for a in range(1, d):
            for b in range(a + 1, d + 1):
                lhs = Fraction(S[a] ** 2, n[a]) + Fraction((S[b] - S[a]) ** 2, n[b] - n[a]) - Fraction(S[b] ** 2, n[b])
                assert lhs == T(a, b)
        K = min(4, d)
        F = {(1, b): Fraction(S[b] ** 2, n[b]) for b in range(1, d + 1)}
        G = {(1, b): Fraction(0) for b in range(1, d + 1)}
        for j in range(2, K + 1):
            for b in range(j, d + 1):
                fv = [(F[(j - 1, a)] + Fraction((S[b] - S[a]) ** 2, n[b] - n[a]), a) for a in range(j - 1, b)]
                gv = [(G[(j - 1, a)] + T(a, b), a) for a in range(j - 1, b)]
                fbest = max(v for v, _ in fv)
                gbest = max(v for v, _ in gv)
                assert [a for v, a in fv if v == fbest] == [a for v, a in gv if v == gbest]
                F[(j, b)], G[(j, b)] = fbest, gbest
                assert gbest == fbest - Fraction(S[b] ** 2, n[b])
