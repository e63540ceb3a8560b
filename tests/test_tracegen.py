"""The seeded input generator (CPU side): deterministic, shardable by row, and
shaped like the paper's workloads."""
import numpy as np
import pytest

import tracegen as G


@pytest.mark.parametrize("name", ["C1", "C2", "C3", "C4", "C5"])
def test_deterministic_and_shardable(name):
    sp = G.spec(name)
    a = G.generate_np(sp, 1000, 5000)
    b = G.generate_np(G.spec(name), 1000, 5000)
    for x, y in zip(a, b):
        if x is not None:
            assert np.array_equal(x, y)
    # rows [1000, 6000) == rows [1000, 3000) ++ [3000, 6000)
    c1 = G.generate_np(sp, 1000, 2000)
    c2 = G.generate_np(sp, 3000, 3000)
    assert np.array_equal(a[0], np.concatenate([c1[0], c2[0]]))
    assert np.array_equal(a[1], np.concatenate([c1[1], c2[1]]))
    assert a[0].max() < sp.n_kernels


def test_c1_shape():
    sp = G.spec("C1")
    kid, t, met = G.generate_np(sp)
    assert len(kid) == 10_000 and met is None
    counts = np.bincount(kid, minlength=20)
    assert counts.min() == counts.max() == 500          # uniform kernel frequency
    for k in range(20):                                  # bimodal: two separated modes
        x = np.sort(t[kid == k]).astype(float)
        gap = np.argmax(np.diff(x))
        assert x[gap + 1] / x[gap] > 1.3
        assert 2000 * 0.8 < x.min() and x.max() < 150_000 * 1.2


def test_c3_metrics_and_heavy_tail():
    sp = G.spec("C3")
    kid, t, met = G.generate_np(sp, 0, 400_000)
    assert met.shape == (12, 400_000)
    rates = met[sp.mclamp == 1]
    assert rates.min() >= 0.0 and rates.max() <= 1.0
    counts = np.bincount(kid, minlength=sp.n_kernels)
    assert counts.max() > 50 * np.median(counts[counts > 0])   # Zipf frequencies
    x = t.astype(float)
    assert x.max() < 2 ** 32 and np.mean(x > 10 * np.median(x)) > 0.01   # heavy tail
