"""Shared helpers of the parity tests: compare a CUDA plan with an oracle plan."""
import numpy as np

Z95 = 1.959963984540054       # scipy.stats.norm.ppf(0.975), passed explicitly to both sides
REL = 1e-9                    # north_star: fp64 estimates and bounds agree to 1e-9 relative

INT_FIELDS = ("kernel_id", "ordinal", "lo_ns", "hi_ns", "n", "sum_ns", "m", "census")


def rel_close(a, b, rel=REL):
    a = np.asarray(a, np.float64)
    b = np.asarray(b, np.float64)
    return np.all(np.abs(a - b) <= rel * np.maximum(np.abs(b), 1e-300))


def assert_plans_equal(got: dict, ref: dict, metrics: bool = False):
    cl = got["clusters"]
    assert len(cl) == len(ref["n"]), (len(cl), len(ref["n"]))
    for f in INT_FIELDS:
        g = cl[f].astype(np.int64)
        r = ref[f].astype(np.int64)
        if not np.array_equal(g, r):
            bad = np.nonzero(g != r)[0][:5]
            raise AssertionError(f"cluster field {f} differs at {bad}: gpu {g[bad]} oracle {r[bad]}")
    assert rel_close(cl["mean_ns"], ref["mean_ns"])
    assert rel_close(cl["std_ns"], ref["std_ns"])
    assert np.array_equal(got["sample_row"], ref["sample_row"]), "sample rows differ"
    assert np.array_equal(got["sample_cluster"], ref["sample_cluster"]), "sample clusters differ"
    assert rel_close(got["sample_weight"], ref["sample_weight"])
    assert got["true_total_ns"] == ref["true_total_ns"]
    assert rel_close(got["est_total_ns"], ref["est_total_ns"])
    if ref["bound"] == 0:
        assert got["bound"] == 0
    else:
        assert rel_close(got["bound"], ref["bound"])
    assert got["z"] == ref["z"] and got["eps"] == ref["eps"]
    if metrics:
        assert rel_close(got["est_metric"], ref["est_metric"])
    if ref.get("true_metric") is not None:   # metric_bounds (R28)
        assert got["true_metric"] is not None and got["bound_metric"] is not None
        assert rel_close(got["true_metric"], ref["true_metric"])
        gb, rb = np.asarray(got["bound_metric"]), np.asarray(ref["bound_metric"])
        assert np.array_equal(np.isinf(gb), np.isinf(rb)) and np.array_equal(gb == 0, rb == 0)
        fin = np.isfinite(rb) & (rb != 0)
        assert rel_close(gb[fin], rb[fin])
    elif "true_metric" in ref:
        assert got.get("true_metric") is None
