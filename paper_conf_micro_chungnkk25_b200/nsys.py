"""Trace ingestion front end: an Nsight Systems export
(``nsys export --type sqlite``) -> the ``(kernel_id, exec_ns)`` columns that
``stem_root_plan`` takes.

The paper profiles execution times with NSYS and groups kernel
calls by name (reading R19: a dense u32 id per kernel name, launch
configuration ignored unless asked for).  This module reads the kernel activity
table of the export::

    CUPTI_ACTIVITY_KIND_KERNEL(start, end, shortName, demangledName, gridX, gridY,
                               gridZ, blockX, blockY, blockZ, ...)
    StringIds(id, value)

orders the invocations by start time (the trace order the plan's row indices
refer to), dictionary-encodes the grouping key into dense ids 0..K-1 (in order
of first appearance) and returns ``exec_ns = end - start`` as u32 (R20: a call
of 2^32 ns or longer is rejected, as the C ABI would with STEM_E_RANGE).

It is the step before the hot path: host-side table reading and encoding only,
nothing of the method's arithmetic."""
import sqlite3

import numpy as np

_KEYS = ("shortName", "demangledName", "mangledName")


def load_nsys_sqlite(path: str, key: str = "shortName", by_launch_config: bool = False, device: int | None = None):
    """Read one export.  Returns (kernel_id u32[n], exec_ns u32[n], names list[K]).

    key: the StringIds column naming a kernel (shortName, demangledName, mangledName).
    by_launch_config: also split groups by (grid, block) dimensions.
    device: keep only the kernels of this deviceId (None: all)."""
    if key not in _KEYS:
        raise ValueError(f"key must be one of {_KEYS}")
    con = sqlite3.connect(f"file:{path}?mode=ro", uri=True)
    try:
        cols = {r[1] for r in con.execute("PRAGMA table_info(CUPTI_ACTIVITY_KIND_KERNEL)")}
        if not cols:
            raise ValueError(f"{path}: no CUPTI_ACTIVITY_KIND_KERNEL table (was the trace taken with CUDA tracing?)")
        if key not in cols:
            raise ValueError(f"{path}: CUPTI_ACTIVITY_KIND_KERNEL has no {key} column")
        sel = ["k.start", "k.end", f"k.{key}"]
        dims = ("gridX", "gridY", "gridZ", "blockX", "blockY", "blockZ")
        if by_launch_config:
            missing = [d for d in dims if d not in cols]
            if missing:
                raise ValueError(f"{path}: missing launch-configuration columns {missing}")
            sel += [f"k.{d}" for d in dims]
        where = ""
        args = ()
        if device is not None:
            where = " WHERE k.deviceId = ?"
            args = (int(device),)
        rows = con.execute(f"SELECT {', '.join(sel)} FROM CUPTI_ACTIVITY_KIND_KERNEL k{where} "
                           f"ORDER BY k.start, k.rowid", args).fetchall()
        strings = dict(con.execute("SELECT id, value FROM StringIds").fetchall())
    finally:
        con.close()
    if not rows:
        raise ValueError(f"{path}: no kernel invocations")
    a = np.asarray(rows, dtype=np.int64)
    dur = a[:, 1] - a[:, 0]
    if np.any(dur < 0):
        raise ValueError("an invocation ends before it starts")
    if np.any(dur >= 2 ** 32):
        raise ValueError("an invocation lasts 2^32 ns or longer (exec_ns is u32, reading R20)")
    keys = a[:, 2:]
    # dense ids in order of first appearance
    uniq, first, inv = np.unique(keys, axis=0, return_index=True, return_inverse=True)
    order = np.argsort(first, kind="stable")
    rank = np.empty(len(order), np.int64)
    rank[order] = np.arange(len(order))
    kernel_id = rank[inv.reshape(-1)].astype(np.uint32)
    names = []
    for u in uniq[order]:
        nm = strings.get(int(u[0]), f"<string {int(u[0])}>")
        if by_launch_config:
            nm += " <<<({},{},{}),({},{},{})>>>".format(*[int(x) for x in u[1:]])
        names.append(nm)
    return kernel_id, dur.astype(np.uint32), names
