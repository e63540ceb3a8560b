"""The sampling-quality harness (tools/quality.py) on a
C2-shaped trace: the library's plans meet their stated error bound (Eq. 5,
P:L158) the way the paper measures it (Eq. 1 error, harmonic-mean speedup,
P:L252-258), and beat uniform random sampling at equal or better speedup."""
import os
import sys

import pytest

sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tools"))


@pytest.mark.gpu
def test_quality_harness_c2():
    import quality
    res = quality.run("C2", n=200_000, n_seeds=24, eps_list=(0.03, 0.25))
    m = res["methods"]
    eps = res["eps"]
    for name in ("stem+root", "stem", "per-kernel", "per-leaf", "lloyd"):
        r = m[name]
        assert r["mean_error_pct"] < 100 * eps, (name, r)
        assert r["coverage_of_eps"] >= 0.9, (name, r)
        assert r["mean_bound_pct"] <= 100 * eps + 1e-9, (name, r)
        assert r["coverage_of_bound"] >= 0.75, (name, r)    # a 95% CLT interval over 24 seeds
    # joint solve never needs more samples than independent per-leaf Eq. 3
    assert m["stem+root"]["mean_samples"] <= m["per-leaf"]["mean_samples"]
    # uniform random at 0.1% (the paper's baseline) is far less accurate
    assert m["random-0.001"]["mean_error_pct"] > m["stem+root"]["mean_error_pct"]
    # a looser bound needs fewer samples (Fig. 11)
    sw = res["eps_sweep"]
    assert sw["0.03"]["mean_samples"] >= sw["0.25"]["mean_samples"]
    assert sw["0.03"]["hmean_speedup"] <= sw["0.25"]["hmean_speedup"]
