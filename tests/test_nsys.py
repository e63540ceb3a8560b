"""Nsight Systems export ingestion: the kernel table of a
synthetic export in the nsys SQLite schema becomes dense kernel ids grouped by
name and integer-ns durations, ordered by start time."""
import sqlite3

import numpy as np
import pytest

from paper_conf_micro_chungnkk25_b200 import nsys


def _export(path, calls, strings):
    con = sqlite3.connect(path)
    con.execute("CREATE TABLE StringIds (id INTEGER PRIMARY KEY, value TEXT NOT NULL)")
    con.execute("CREATE TABLE CUPTI_ACTIVITY_KIND_KERNEL (start INTEGER NOT NULL, end INTEGER NOT NULL, "
                "deviceId INTEGER, streamId INTEGER, correlationId INTEGER, demangledName INTEGER, "
                "shortName INTEGER, mangledName INTEGER, gridX INTEGER, gridY INTEGER, gridZ INTEGER, "
                "blockX INTEGER, blockY INTEGER, blockZ INTEGER)")
    con.executemany("INSERT INTO StringIds VALUES (?, ?)", list(strings.items()))
    con.executemany("INSERT INTO CUPTI_ACTIVITY_KIND_KERNEL VALUES (?,?,?,?,?,?,?,?,?,?,?,?,?,?)", calls)
    con.commit()
    con.close()


def _calls(rng, n):
    # (start, end, dev, stream, corr, demangled, short, mangled, grid..., block...)
    out, t = [], 1_000
    shorts = [10, 11, 12]        # gemm, softmax, gemm (same short name as 10 via string id 10)
    for i in range(n):
        s = int(rng.integers(0, 3))
        dur = int(rng.integers(2_000, 90_000))
        grid = (128, 1, 1) if i % 2 else (256, 1, 1)
        out.append((t, t + dur, i % 2, 7, i, 20 + s, shorts[s], 30 + s) + grid + (256, 1, 1))
        t += dur + int(rng.integers(0, 500))
    return out


def test_nsys_ingestion(tmp_path):
    rng = np.random.default_rng(0)
    calls = _calls(rng, 500)
    strings = {10: "gemm", 11: "softmax", 12: "layernorm", 20: "void gemm<128>(float*)", 21: "softmax_kernel",
               22: "ln_fwd", 30: "_Z4gemm", 31: "_Z7softmax", 32: "_Z2ln"}
    path = str(tmp_path / "trace.sqlite")
    shuffled = [calls[i] for i in rng.permutation(len(calls))]   # table order is not trace order
    _export(path, shuffled, strings)
    kid, t, names = nsys.load_nsys_sqlite(path)
    assert kid.dtype == np.uint32 and t.dtype == np.uint32 and len(kid) == len(calls)
    exp_t = np.array([c[1] - c[0] for c in calls], np.uint32)
    assert np.array_equal(t, exp_t)                                  # ordered by start
    exp_names = []
    for c in calls:
        nm = strings[c[6]]
        if nm not in exp_names:
            exp_names.append(nm)
    assert names == exp_names                                        # first-appearance order
    assert np.array_equal(np.array(names)[kid], np.array([strings[c[6]] for c in calls]))
    # by launch configuration: more groups, each a (name, grid, block)
    kid2, _, names2 = nsys.load_nsys_sqlite(path, by_launch_config=True)
    assert len(names2) == 2 * len(names) and kid2.max() == len(names2) - 1
    # one device only
    kid3, t3, _ = nsys.load_nsys_sqlite(path, device=1)
    assert len(kid3) == sum(1 for c in calls if c[2] == 1)


def test_nsys_rejects_long_calls(tmp_path):
    path = str(tmp_path / "long.sqlite")
    _export(path, [(0, 2 ** 32, 0, 0, 0, 1, 1, 1, 1, 1, 1, 1, 1, 1)], {1: "k"})
    with pytest.raises(ValueError, match="2\\^32"):
        nsys.load_nsys_sqlite(path)
    with pytest.raises(ValueError):
        nsys.load_nsys_sqlite(path, key="bogus")


@pytest.mark.gpu
def test_nsys_trace_plans_like_the_oracle(tmp_path):
    import oracle as O
    import paper_conf_micro_chungnkk25_b200 as sr
    rng = np.random.default_rng(1)
    calls = _calls(rng, 20_000)
    path = str(tmp_path / "t.sqlite")
    _export(path, calls, {10: "gemm", 11: "softmax", 12: "layernorm"})
    kid, t, names = nsys.load_nsys_sqlite(path)
    z = 1.959963984540054
    ctx = sr.Context(0)
    got = ctx.plan(kid, t, len(names), eps=0.05, z=z, seed=3)
    ctx.close()
    ref = O.plan(kid, t, len(names), eps=0.05, z=z, seed=3)
    assert np.array_equal(got["sample_row"], ref["sample_row"])
    assert np.array_equal(got["clusters"]["n"].astype(np.int64), ref["n"].astype(np.int64))
