"""STEM+ROOT oracle -- TEST INFRASTRUCTURE ONLY.

A plain single-threaded C implementation (``stemroot_oracle.c``) of the
sampling-plan hot path, written from PAPER.md (Chung et al., MICRO'25) and
the readings in DESIGN.md §3.  Only ``tests/``, ``__graft_entry__.smoke()``
and ``bench.py`` (its ``cpu_baseline`` leg and ``--impl reference``) may
import this package.  It shares no code with the CUDA library in
``paper_conf_micro_chungnkk25_b200/``; neither imports the other.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "stemroot_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")

OR_OK, OR_E_INVAL, OR_E_RANGE, OR_E_NOMEM, OR_E_LIMIT = 0, -1, -2, -3, -6


def build(force: bool = False) -> str:
    """Compile liboracle.so with gcc (-ffp-contract=off keeps fp64 order)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < max(
            os.path.getmtime(_SRC), os.path.getmtime(os.path.join(_HERE, "stemroot_oracle.h"))):
        subprocess.check_call([
            "gcc", "-O2", "-std=c11", "-ffp-contract=off", "-fno-fast-math", "-fPIC", "-shared",
            "-o", _LIB, _SRC, "-lm"])
    return _LIB


class _Opts(C.Structure):
    _fields_ = [("seed", C.c_uint64), ("z", C.c_double), ("scope", C.c_int), ("root", C.c_int),
                ("clamp_in_split", C.c_int), ("census_cap", C.c_int), ("split", C.c_int),
                ("metric_bounds", C.c_int), ("kmeans_k", C.c_int)]


class _Plan(C.Structure):
    _fields_ = [
        ("n_clusters", C.c_uint64),
        ("kernel_id", C.POINTER(C.c_uint32)), ("ordinal", C.POINTER(C.c_uint32)),
        ("lo_ns", C.POINTER(C.c_uint32)), ("hi_ns", C.POINTER(C.c_uint32)),
        ("n", C.POINTER(C.c_uint64)), ("sum_ns", C.POINTER(C.c_uint64)), ("m", C.POINTER(C.c_uint64)),
        ("mean_ns", C.POINTER(C.c_double)), ("std_ns", C.POINTER(C.c_double)),
        ("census", C.POINTER(C.c_uint8)),
        ("n_samples", C.c_uint64),
        ("sample_row", C.POINTER(C.c_uint32)), ("sample_cluster", C.POINTER(C.c_uint32)),
        ("sample_weight", C.POINTER(C.c_double)),
        ("est_total_ns", C.c_double), ("true_total_ns", C.c_uint64),
        ("bound", C.c_double), ("eps", C.c_double), ("z", C.c_double),
        ("n_metrics", C.c_uint32), ("est_metric", C.POINTER(C.c_double)),
        ("ssum", C.c_double), ("max_depth", C.c_uint32),
        ("true_metric", C.POINTER(C.c_double)), ("bound_metric", C.POINTER(C.c_double)),
    ]


_lib = None


def lib():
    global _lib
    if _lib is None:
        _lib = C.CDLL(build())
        u32p, u64p, dp = C.POINTER(C.c_uint32), C.POINTER(C.c_uint64), C.POINTER(C.c_double)
        _lib.or_plan_build.argtypes = [C.c_uint64, C.c_uint32, u32p, u32p, C.c_uint32, dp, C.c_double,
                                       C.POINTER(_Opts), C.POINTER(C.POINTER(_Plan))]
        _lib.or_plan_build.restype = C.c_int
        _lib.or_plan_free.argtypes = [C.POINTER(_Plan)]
        _lib.or_philox4x32_10.argtypes = [u32p, u32p, u32p]
        _lib.or_best_cut.argtypes = [u32p, C.c_uint64]
        _lib.or_best_cut.restype = C.c_uint64
        _lib.or_lloyd_cut.argtypes = [u32p, C.c_uint64, C.POINTER(C.c_uint32)]
        _lib.or_lloyd_cut.restype = C.c_uint64
        _lib.or_kmpp_cut.argtypes = [u32p, C.c_uint64, C.c_uint64, C.POINTER(C.c_uint32), C.POINTER(C.c_uint32),
                                     C.POINTER(C.c_uint32)]
        _lib.or_kmpp_cut.restype = C.c_uint64
        _lib.or_kmeans_cuts.argtypes = [u32p, C.c_uint64, C.c_uint32, u64p]
        _lib.or_kmeans_cuts.restype = C.c_uint32
        _lib.or_eq3_m.argtypes = [C.c_uint64, C.c_uint64, C.c_uint64, C.c_uint64, C.c_double, C.c_double, C.c_int]
        _lib.or_eq3_m.restype = C.c_double
        _lib.or_eq6_m.argtypes = [C.c_uint32, dp, dp, C.c_double, C.c_double, C.c_double, dp]
        _lib.or_root_decide.argtypes = [u32p, C.c_uint64, C.c_double, C.c_double, C.c_int, dp, dp, u64p]
        _lib.or_root_decide.restype = C.c_int
        _lib.or_exact_sum.argtypes = [dp, C.c_uint64]
        _lib.or_exact_sum.restype = C.c_double
        _lib.or_exact_sum_signed.argtypes = [dp, C.c_uint64]
        _lib.or_exact_sum_signed.restype = C.c_double
        _lib.or_u128_to_double.argtypes = [C.c_uint64, C.c_uint64]
        _lib.or_u128_to_double.restype = C.c_double
        _lib.or_z_from_conf.argtypes = [C.c_double]
        _lib.or_z_from_conf.restype = C.c_double
    return _lib


def _u32(a):
    return np.ascontiguousarray(a, dtype=np.uint32)


def _ptr(a, ct):
    return a.ctypes.data_as(C.POINTER(ct))


class OracleError(RuntimeError):
    def __init__(self, status):
        super().__init__(f"oracle status {status}")
        self.status = status


def plan(kernel_id, exec_ns, n_kernels, eps=0.05, z=1.959963984540054, seed=0, scope=0, root=1,
         clamp_in_split=1, census_cap=0, metrics=None, split=0, metric_bounds=0, kmeans_k=3) -> dict:
    """Full sampling plan (§3).  Returns numpy arrays + scalars."""
    kid = _u32(kernel_id)
    t = _u32(exec_ns)
    n = kid.shape[0]
    if metrics is not None:
        met = np.ascontiguousarray(metrics, dtype=np.float64)
        nm = met.shape[0]
        metp = _ptr(met, C.c_double)
    else:
        nm, metp = 0, None
    o = _Opts(seed, z, scope, root, clamp_in_split, census_cap, split, int(metric_bounds), int(kmeans_k))
    out = C.POINTER(_Plan)()
    st = lib().or_plan_build(n, n_kernels, _ptr(kid, C.c_uint32), _ptr(t, C.c_uint32), nm, metp, eps,
                             C.byref(o), C.byref(out))
    if st != OR_OK:
        raise OracleError(st)
    p = out.contents
    L, S = p.n_clusters, p.n_samples

    def arr(ptr, cnt, dt):
        return np.ctypeslib.as_array(ptr, shape=(cnt,)).astype(dt, copy=True) if cnt else np.zeros(0, dt)

    res = dict(
        kernel_id=arr(p.kernel_id, L, np.uint32), ordinal=arr(p.ordinal, L, np.uint32),
        lo_ns=arr(p.lo_ns, L, np.uint32), hi_ns=arr(p.hi_ns, L, np.uint32),
        n=arr(p.n, L, np.uint64), sum_ns=arr(p.sum_ns, L, np.uint64), m=arr(p.m, L, np.uint64),
        mean_ns=arr(p.mean_ns, L, np.float64), std_ns=arr(p.std_ns, L, np.float64),
        census=arr(p.census, L, np.uint8),
        sample_row=arr(p.sample_row, S, np.uint32), sample_cluster=arr(p.sample_cluster, S, np.uint32),
        sample_weight=arr(p.sample_weight, S, np.float64),
        est_total_ns=p.est_total_ns, true_total_ns=int(p.true_total_ns), bound=p.bound, eps=p.eps, z=p.z,
        est_metric=arr(p.est_metric, p.n_metrics, np.float64), ssum=p.ssum, max_depth=int(p.max_depth),
        true_metric=arr(p.true_metric, p.n_metrics, np.float64) if p.true_metric else None,
        bound_metric=arr(p.bound_metric, p.n_metrics, np.float64) if p.bound_metric else None,
    )
    lib().or_plan_free(out)
    return res


def philox4x32_10(ctr, key):
    c = _u32(ctr)
    k = _u32(key)
    o = np.zeros(4, np.uint32)
    lib().or_philox4x32_10(_ptr(c, C.c_uint32), _ptr(k, C.c_uint32), _ptr(o, C.c_uint32))
    return [int(x) for x in o]


def lloyd_cut(t_sorted):
    """Lloyd's k-means (k = 2) cut of sorted times and its assignment steps (reading R26)."""
    t = _u32(t_sorted)
    it = C.c_uint32(0)
    k = int(lib().or_lloyd_cut(_ptr(t, C.c_uint32), t.shape[0], C.byref(it)))
    return k, int(it.value)


def kmpp_cut(t_sorted, seed):
    """Lloyd's k-means (k = 2) from k-means++ seeds (reading R27): (cut, c1, c2, steps)."""
    t = _u32(t_sorted)
    c1, c2, it = C.c_uint32(0), C.c_uint32(0), C.c_uint32(0)
    k = int(lib().or_kmpp_cut(_ptr(t, C.c_uint32), t.shape[0], seed & 0xFFFFFFFFFFFFFFFF, C.byref(c1),
                              C.byref(c2), C.byref(it)))
    return k, int(c1.value), int(c2.value), int(it.value)


def kmeans_cuts(t_sorted, k):
    """Exact optimal 1-D k-means cuts of sorted times (reading R29): list of row cuts."""
    t = _u32(t_sorted)
    out = np.zeros(16, np.uint64)
    g = int(lib().or_kmeans_cuts(_ptr(t, C.c_uint32), t.shape[0], k, _ptr(out, C.c_uint64)))
    return [int(x) for x in out[:max(g - 1, 0)]]


def best_cut(t_sorted) -> int:
    t = _u32(t_sorted)
    return int(lib().or_best_cut(_ptr(t, C.c_uint32), t.shape[0]))


def eq3_m(n, S, Q, eps, z, clamp=1) -> float:
    return lib().or_eq3_m(n, S, Q & ((1 << 64) - 1), Q >> 64, eps, z, clamp)


def eq6_m(mu, V, T, eps, z):
    mu = np.ascontiguousarray(mu, dtype=np.float64)
    V = np.ascontiguousarray(V, dtype=np.float64)
    out = np.zeros_like(mu)
    lib().or_eq6_m(mu.shape[0], _ptr(mu, C.c_double), _ptr(V, C.c_double), float(T), eps, z,
                   _ptr(out, C.c_double))
    return out


def root_decide(t_sorted, eps, z, clamp=1):
    t = _u32(t_sorted)
    to, tn, cut = C.c_double(), C.c_double(), C.c_uint64()
    s = lib().or_root_decide(_ptr(t, C.c_uint32), t.shape[0], eps, z, clamp, C.byref(to), C.byref(tn),
                             C.byref(cut))
    return bool(s), to.value, tn.value, int(cut.value)


def exact_sum(x) -> float:
    a = np.ascontiguousarray(x, dtype=np.float64)
    return lib().or_exact_sum(_ptr(a, C.c_double), a.shape[0])


def exact_sum_signed(x) -> float:
    a = np.ascontiguousarray(x, dtype=np.float64)
    return lib().or_exact_sum_signed(_ptr(a, C.c_double), a.shape[0])


def u128_to_double(v: int) -> float:
    return lib().or_u128_to_double(v & ((1 << 64) - 1), v >> 64)


def z_from_conf(conf: float) -> float:
    return lib().or_z_from_conf(conf)
