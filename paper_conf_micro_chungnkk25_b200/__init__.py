"""B200-native STEM+ROOT sampling-plan builder: thin Python binding.

Argument marshalling only -- every step of the plan runs in the CUDA kernels
of ``lib/libstemroot.so`` behind the C ABI declared in ``include/stemroot.h``
(same function names).  There is no CPU path: if the library is missing or
cannot find a GPU, every call raises.

    import paper_conf_micro_chungnkk25_b200 as sr
    ctx = sr.Context(0)
    plan = ctx.plan(kernel_id, exec_ns, n_kernels, eps=0.05, conf=0.95)

``kernel_id`` / ``exec_ns`` are uint32 data either as CUDA tensors (int32 or
uint32 dtype, bytes reinterpreted; other dtypes raise TypeError) on the
context's device, or as host arrays (4-byte integers viewed, other integer
arrays range-checked and converted; the library copies them in).  ``metrics``
is float64, shape (n_metrics, n) or (n,).  PAPER.md citations: see
include/stemroot.h.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_ROOT = os.path.dirname(_HERE)
_CSRC = os.path.join(_HERE, "csrc")
# STEMROOT_LIB: another build of the same sources (the bounds-checked -DSR_CHECK
# build of tests/test_gpu_checked.py); default the in-tree libstemroot.so
LIB_PATH = os.environ.get("STEMROOT_LIB") or os.path.join(_HERE, "lib", "libstemroot.so")
HEADER = os.path.join(_ROOT, "include", "stemroot.h")
SOURCES = ["capi.cu", "sort.cu", "root.cu", "stem.cu", "dist.cu", "metric.cu", "kmeans.cu"]
NVCC_FLAGS = ["-O3", "-std=c++17", "-gencode", "arch=compute_100a,code=sm_100a", "-lineinfo", "--fmad=false",
              "--extended-lambda", "-Xcompiler", "-fPIC,-fvisibility=hidden", "-shared"]

STEM_OK, STEM_E_INVAL, STEM_E_RANGE, STEM_E_NOMEM, STEM_E_CUDA, STEM_E_NCCL, STEM_E_LIMIT, STEM_E_STATE = \
    0, -1, -2, -3, -4, -5, -6, -7


def _nccl_include():
    import glob
    import sys
    for sp in sys.path:
        hit = glob.glob(os.path.join(sp, "nvidia", "nccl", "include", "nccl.h"))
        if hit:
            return os.path.dirname(hit[0])
    for p in ("/usr/include", "/usr/local/cuda/include"):
        if os.path.exists(os.path.join(p, "nccl.h")):
            return p
    raise RuntimeError("nccl.h not found (the NCCL headers are needed to build dist.cu)")


def build(force: bool = False, verbose: bool = False) -> str:
    """Compile libstemroot.so for sm_100a in-tree (nvcc cross-compiles without a GPU)."""
    srcs = [os.path.join(_CSRC, s) for s in SOURCES]
    deps = srcs + [os.path.join(_CSRC, h) for h in os.listdir(_CSRC) if h.endswith((".cuh", ".h"))] + [HEADER]
    if not force and os.path.exists(LIB_PATH) and os.path.getmtime(LIB_PATH) >= max(map(os.path.getmtime, deps)):
        return LIB_PATH
    os.makedirs(os.path.dirname(LIB_PATH), exist_ok=True)
    extra = os.environ.get("SR_EXTRA_NVCC", "").split()   # A/B builds only (tools/ab_build.sh)
    cmd = ["nvcc"] + NVCC_FLAGS + extra + ["-I", _nccl_include()] + (["-Xptxas", "-v"] if verbose else []) + \
        ["-o", LIB_PATH] + srcs + ["-ldl"]
    subprocess.check_call(cmd, cwd=_CSRC)
    return LIB_PATH


# ------------------------------------------------------------------ ABI structs (mirror stemroot.h)
class stem_trace(C.Structure):
    _fields_ = [("n", C.c_uint64), ("n_kernels", C.c_uint32), ("kernel_id", C.c_void_p), ("exec_ns", C.c_void_p),
                ("n_metrics", C.c_uint32), ("metrics", C.c_void_p), ("device", C.c_int)]


class stem_opts(C.Structure):
    _fields_ = [("seed", C.c_uint64), ("z", C.c_double), ("scope", C.c_int), ("root", C.c_int),
                ("clamp_in_split", C.c_int), ("census_cap", C.c_int), ("split", C.c_int),
                ("metric_bounds", C.c_int), ("kmeans_k", C.c_int), ("stream", C.c_void_p)]


class stem_cluster(C.Structure):
    _fields_ = [("kernel_id", C.c_uint32), ("ordinal", C.c_uint32), ("lo_ns", C.c_uint32), ("hi_ns", C.c_uint32),
                ("n", C.c_uint64), ("sum_ns", C.c_uint64), ("mean_ns", C.c_double), ("std_ns", C.c_double),
                ("m", C.c_uint64), ("census", C.c_uint32), ("reserved", C.c_uint32)]


CLUSTER_DTYPE = np.dtype([("kernel_id", "<u4"), ("ordinal", "<u4"), ("lo_ns", "<u4"), ("hi_ns", "<u4"),
                          ("n", "<u8"), ("sum_ns", "<u8"), ("mean_ns", "<f8"), ("std_ns", "<f8"), ("m", "<u8"),
                          ("census", "<u4"), ("reserved", "<u4")])
assert CLUSTER_DTYPE.itemsize == C.sizeof(stem_cluster)


class stem_plan(C.Structure):
    _fields_ = [("n_clusters", C.c_uint64), ("clusters", C.POINTER(stem_cluster)), ("n_samples", C.c_uint64),
                ("sample_row", C.POINTER(C.c_uint32)), ("sample_cluster", C.POINTER(C.c_uint32)),
                ("sample_weight", C.POINTER(C.c_double)), ("est_total_ns", C.c_double),
                ("true_total_ns", C.c_uint64), ("bound", C.c_double), ("eps", C.c_double), ("z", C.c_double),
                ("n_metrics", C.c_uint32), ("est_metric", C.POINTER(C.c_double)),
                ("true_metric", C.POINTER(C.c_double)), ("bound_metric", C.POINTER(C.c_double))]


class stem_device_plan(C.Structure):
    _fields_ = [("n_clusters", C.c_uint64), ("n_samples", C.c_uint64), ("clusters", C.c_void_p),
                ("sample_row", C.c_void_p), ("sample_cluster", C.c_void_p), ("sample_weight", C.c_void_p),
                ("est_total_ns", C.c_double), ("bound", C.c_double), ("eps", C.c_double), ("z", C.c_double),
                ("true_total_ns", C.c_uint64), ("n_metrics", C.c_uint32), ("est_metric", C.POINTER(C.c_double)),
                ("true_metric", C.POINTER(C.c_double)), ("bound_metric", C.POINTER(C.c_double))]


class stem_stats(C.Structure):
    _fields_ = [("key_bits", C.c_uint32), ("sort_passes", C.c_uint32), ("levels", C.c_uint32),
                ("kernel_launches", C.c_uint32), ("active_rows", C.c_uint64), ("n_clusters", C.c_uint64),
                ("n_samples", C.c_uint64), ("ssum", C.c_double), ("pack_bits", C.c_uint32),
                ("ambiguous_samples", C.c_uint32), ("coarse_bases", C.c_uint32), ("reserved0", C.c_uint32),
                ("split_chunks", C.c_uint64), ("split_scanned", C.c_uint64), ("owned_rows", C.c_uint64),
                ("world", C.c_uint32), ("fused_exchange", C.c_uint32), ("value_levels", C.c_uint32),
                ("value_groups", C.c_uint64), ("value_count", C.c_uint64)]


class stem_stage_time(C.Structure):
    _fields_ = [("name", C.c_char * 24), ("ms", C.c_double), ("bytes", C.c_uint64), ("launches", C.c_uint32),
                ("count", C.c_uint32)]


EXPORTS = ["stem_default_opts", "stem_ctx_create", "stem_ctx_destroy", "stem_root_plan_ctx", "stem_root_plan",
           "stem_ctx_device_plan", "stem_ctx_stats", "stem_plan_free", "stem_strerror", "stem_z_from_conf",
           "stem_ctx_enable_timing", "stem_ctx_stage_times", "stem_comm_nccl_unique_id", "stem_comm_init_nccl",
           "stem_comm_init_loopback", "stem_comm_destroy", "stem_owner_ranges", "stem_root_plan_dist"]

_lib = None


def lib():
    """Load libstemroot.so (raises if it was not built: there is no fallback)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise RuntimeError(f"{LIB_PATH} missing: run __graft_entry__.build() (no CPU fallback exists)")
        L = C.CDLL(LIB_PATH)
        P = C.POINTER
        L.stem_default_opts.argtypes = [P(stem_opts)]
        L.stem_ctx_create.argtypes = [C.c_int, P(C.c_void_p)]
        L.stem_ctx_destroy.argtypes = [C.c_void_p]
        L.stem_ctx_destroy.restype = None
        L.stem_root_plan_ctx.argtypes = [C.c_void_p, P(stem_trace), C.c_double, C.c_double, P(stem_opts),
                                         P(P(stem_plan))]
        L.stem_root_plan.argtypes = [P(stem_trace), C.c_double, C.c_double, P(stem_opts), P(P(stem_plan))]
        L.stem_ctx_device_plan.argtypes = [C.c_void_p, P(stem_device_plan)]
        L.stem_ctx_stats.argtypes = [C.c_void_p, P(stem_stats)]
        L.stem_plan_free.argtypes = [P(stem_plan)]
        L.stem_plan_free.restype = None
        L.stem_strerror.argtypes = [C.c_int]
        L.stem_strerror.restype = C.c_char_p
        L.stem_z_from_conf.argtypes = [C.c_double, P(C.c_double)]
        L.stem_ctx_enable_timing.argtypes = [C.c_void_p, C.c_int]
        L.stem_ctx_stage_times.argtypes = [C.c_void_p, P(stem_stage_time), C.c_uint32, P(C.c_uint32)]
        L.stem_comm_nccl_unique_id.argtypes = [C.c_void_p]
        L.stem_comm_init_nccl.argtypes = [C.c_void_p, C.c_int, C.c_int, C.c_int, P(C.c_void_p)]
        L.stem_comm_init_loopback.argtypes = [C.c_int, C.c_int, P(C.c_void_p)]
        L.stem_comm_destroy.argtypes = [C.c_void_p]
        L.stem_comm_destroy.restype = None
        L.stem_owner_ranges.argtypes = [P(C.c_uint64), C.c_uint32, C.c_int, P(C.c_uint32)]
        L.stem_root_plan_dist.argtypes = [C.c_void_p, C.c_void_p, P(stem_trace), C.c_uint64, C.c_double,
                                          C.c_double, P(stem_opts), P(P(stem_plan))]
        _lib = L
    return _lib


class StemError(RuntimeError):
    def __init__(self, status: int, where: str):
        super().__init__(f"{where}: {lib().stem_strerror(status).decode()} ({status})")
        self.status = status


def _check(st, where):
    if st != STEM_OK:
        raise StemError(st, where)


def strerror(status: int) -> str:
    return lib().stem_strerror(status).decode()


def z_from_conf(conf: float) -> float:
    z = C.c_double()
    _check(lib().stem_z_from_conf(conf, C.byref(z)), "stem_z_from_conf")
    return z.value


def _arg(x, kind: str, n: int = -1):
    """(pointer, device, keepalive, shape) for a torch tensor or numpy array.

    kind "u32": kernel_id / exec_ns -- torch int32/uint32 (bytes reinterpreted
    as uint32); numpy 4-byte integers are viewed, other integer arrays are
    converted after a range check; anything else raises.  kind "f64": metrics
    -- torch float64 only; numpy arrays are converted to float64.  n >= 0
    checks the trailing dimension (rows)."""
    try:
        import torch
        if isinstance(x, torch.Tensor):
            ok = {"u32": (torch.int32, getattr(torch, "uint32", torch.int32)), "f64": (torch.float64,)}[kind]
            if x.dtype not in ok:
                raise TypeError(f"{'kernel_id/exec_ns' if kind == 'u32' else 'metrics'} tensor must be "
                                f"{' or '.join(str(d) for d in ok)}, got {x.dtype}")
            if not x.is_contiguous():
                raise ValueError("tensor must be contiguous")
            if n >= 0 and (x.dim() == 0 or x.shape[-1] != n):
                raise ValueError(f"expected {n} rows in the last dimension, got shape {tuple(x.shape)}")
            return x.data_ptr(), (x.device.index if x.is_cuda else -1), x, tuple(x.shape)
    except ImportError:
        pass
    a = np.asarray(x)
    if kind == "u32":
        if a.dtype.kind not in "iu":
            raise TypeError(f"kernel_id/exec_ns must be integer arrays, got {a.dtype}")
        if a.dtype.itemsize == 4:
            a = np.ascontiguousarray(a).view(np.uint32)
        else:
            if a.size and (int(a.min()) < 0 or int(a.max()) >= 1 << 32):
                raise ValueError("kernel_id/exec_ns values must fit in uint32")
            a = np.ascontiguousarray(a, dtype=np.uint32)
    else:
        a = np.ascontiguousarray(a, dtype=np.float64)
    if n >= 0 and (a.ndim == 0 or a.shape[-1] != n):
        raise ValueError(f"expected {n} rows in the last dimension, got shape {a.shape}")
    return a.ctypes.data, -1, a, a.shape


def _trace(kernel_id, exec_ns, n_kernels, metrics, allow_empty=False):
    """stem_trace + keepalives from the user's arrays (argument marshalling only)."""
    kp, kdev, k_keep, kshape = _arg(kernel_id, "u32")
    if len(kshape) != 1:
        raise ValueError("kernel_id must be one-dimensional")
    n = int(kshape[0])
    tp, tdev, t_keep, _ = _arg(exec_ns, "u32", n)
    if kdev != tdev:
        raise ValueError("kernel_id and exec_ns must live on the same device")
    nm, mp, m_keep = 0, None, None
    if metrics is not None:
        mp, mdev, m_keep, mshape = _arg(metrics, "f64", n)
        if mdev != kdev:
            raise ValueError("metrics must live with the trace")
        if len(mshape) not in (1, 2):
            raise ValueError("metrics must be (n_metrics, n) or (n,)")
        nm = int(mshape[0]) if len(mshape) == 2 else 1
    if n == 0 and allow_empty:
        kp = tp = mp = None
    tr = stem_trace(n, n_kernels, kp, tp, nm, mp, kdev)
    return tr, kdev, (k_keep, t_keep, m_keep)


def _opts(seed, z, scope, root, clamp_in_split, census_cap, split, metric_bounds, stream, dev, kmeans_k=3):
    if stream is None and dev >= 0:
        import torch
        stream = torch.cuda.current_stream(dev).cuda_stream
    return stem_opts(seed & 0xFFFFFFFFFFFFFFFF, z, scope, int(root), int(clamp_in_split), int(census_cap),
                     int(split), int(metric_bounds), int(kmeans_k), stream or None)


def _plan_to_numpy(p: stem_plan) -> dict:
    L, S = p.n_clusters, p.n_samples
    cl = np.ctypeslib.as_array(C.cast(p.clusters, C.POINTER(C.c_uint8)), shape=(L * CLUSTER_DTYPE.itemsize,)) \
        .view(CLUSTER_DTYPE).copy() if L else np.zeros(0, CLUSTER_DTYPE)

    def arr(ptr, cnt, dt):
        return np.ctypeslib.as_array(ptr, shape=(cnt,)).astype(dt, copy=True) if cnt else np.zeros(0, dt)
    return dict(clusters=cl, sample_row=arr(p.sample_row, S, np.uint32),
                sample_cluster=arr(p.sample_cluster, S, np.uint32), sample_weight=arr(p.sample_weight, S, np.float64),
                est_total_ns=p.est_total_ns, true_total_ns=int(p.true_total_ns), bound=p.bound, eps=p.eps, z=p.z,
                est_metric=arr(p.est_metric, p.n_metrics, np.float64),
                true_metric=arr(p.true_metric, p.n_metrics, np.float64) if p.true_metric else None,
                bound_metric=arr(p.bound_metric, p.n_metrics, np.float64) if p.bound_metric else None)


def owner_ranges(counts, world: int) -> np.ndarray:
    """stem_owner_ranges: first kernel id of every rank's contiguous range (+ n_kernels)."""
    c = np.ascontiguousarray(counts, dtype=np.uint64)
    b = np.zeros(world + 1, np.uint32)
    _check(lib().stem_owner_ranges(c.ctypes.data_as(C.POINTER(C.c_uint64)), len(c), world,
                                   b.ctypes.data_as(C.POINTER(C.c_uint32))), "stem_owner_ranges")
    return b


def nccl_unique_id() -> bytes:
    buf = (C.c_uint8 * 128)()
    _check(lib().stem_comm_nccl_unique_id(buf), "stem_comm_nccl_unique_id")
    return bytes(buf)


class Comm:
    """A stem_comm: NCCL (one process per GPU) or one member of a loopback group."""

    def __init__(self, handle, rank, world):
        self._h, self.rank, self.world = handle, rank, world

    @staticmethod
    def nccl(unique_id: bytes, rank: int, world: int, device: int) -> "Comm":
        h = C.c_void_p()
        buf = (C.c_uint8 * 128).from_buffer_copy(unique_id)
        _check(lib().stem_comm_init_nccl(buf, rank, world, device, C.byref(h)), "stem_comm_init_nccl")
        return Comm(h, rank, world)

    @staticmethod
    def loopback(world: int, device: int = 0) -> list:
        arr = (C.c_void_p * world)()
        _check(lib().stem_comm_init_loopback(world, device, arr), "stem_comm_init_loopback")
        return [Comm(C.c_void_p(arr[r]), r, world) for r in range(world)]

    def close(self):
        if self._h:
            lib().stem_comm_destroy(self._h)
            self._h = C.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


class HostPlan:
    """A library-allocated stem_plan (host memory), freed by close() / stem_plan_free."""

    def __init__(self, ptr):
        self._p = ptr

    @property
    def plan(self):
        return self._p.contents if self._p else None

    def nbytes(self) -> int:
        """bytes of the plan's arrays (what the library copied to the host)"""
        p = self.plan
        if p is None:
            return 0
        nmb = 3 if p.true_metric else 1
        return (int(p.n_clusters) * CLUSTER_DTYPE.itemsize + int(p.n_samples) * (4 + 4 + 8) +
                8 * nmb * int(p.n_metrics) + 8 * 6)

    def to_numpy(self) -> dict:
        return _plan_to_numpy(self.plan)

    def close(self):
        if self._p:
            lib().stem_plan_free(self._p)
            self._p = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


class Context:
    """A stem_ctx: device workspace reused across plans (stem_ctx_create)."""

    def __init__(self, device: int = 0):
        self._h = C.c_void_p()
        _check(lib().stem_ctx_create(device, C.byref(self._h)), "stem_ctx_create")
        self.device = device

    def close(self):
        if self._h:
            lib().stem_ctx_destroy(self._h)
            self._h = C.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def plan(self, kernel_id, exec_ns, n_kernels: int, eps: float = 0.05, conf: float = 0.95, metrics=None,
             seed: int = 0, z: float = 0.0, scope: int = 0, root: bool = True, clamp_in_split: bool = True,
             census_cap: bool = False, stream=None, to_host: bool = True, split: int = 0,
             metric_bounds: bool = False, kmeans_k: int = 3):
        """stem_root_plan_ctx.  Returns the host plan as numpy arrays, or None when to_host=False
        (the plan then stays on the device: see device_plan())."""
        tr, dev, keep = _trace(kernel_id, exec_ns, n_kernels, metrics)
        o = _opts(seed, z, scope, root, clamp_in_split, census_cap, split, metric_bounds, stream, dev, kmeans_k)
        out = C.POINTER(stem_plan)()
        st = lib().stem_root_plan_ctx(self._h, C.byref(tr), eps, conf, C.byref(o),
                                      C.byref(out) if to_host else None)
        _check(st, "stem_root_plan_ctx")
        del keep
        if not to_host:
            return None
        res = _plan_to_numpy(out.contents)
        lib().stem_plan_free(out)
        return res

    def plan_dist(self, comm: "Comm", kernel_id, exec_ns, n_kernels: int, global_row_base: int, eps: float = 0.05,
                  conf: float = 0.95, metrics=None, seed: int = 0, z: float = 0.0, scope: int = 0, root: bool = True,
                  clamp_in_split: bool = True, census_cap: bool = False, stream=None, to_host: bool = True,
                  split: int = 0, metric_bounds: bool = False, kmeans_k: int = 3):
        """stem_root_plan_dist (collective).  Returns the global plan on rank 0, None elsewhere."""
        tr, dev, keep = _trace(kernel_id, exec_ns, n_kernels, metrics, allow_empty=True)
        o = _opts(seed, z, scope, root, clamp_in_split, census_cap, split, metric_bounds, stream, dev, kmeans_k)
        out = C.POINTER(stem_plan)()
        st = lib().stem_root_plan_dist(self._h, comm._h, C.byref(tr), global_row_base, eps, conf, C.byref(o),
                                       C.byref(out) if to_host else None)
        _check(st, "stem_root_plan_dist")
        del keep
        if not to_host or not out:
            return None
        res = _plan_to_numpy(out.contents)
        lib().stem_plan_free(out)
        return res

    def plan_host_raw(self, kernel_id, exec_ns, n_kernels: int, eps: float = 0.05, conf: float = 0.95,
                      metrics=None, comm: "Comm" = None, global_row_base: int = 0, **kw) -> "HostPlan":
        """stem_root_plan_ctx (or _dist with comm) with the host plan kept as the
        library allocated it (no numpy conversion): a HostPlan whose close()
        calls stem_plan_free.  On ranks other than 0 of a dist plan it is empty."""
        opt = {k: kw.pop(k) for k in list(kw) if k in ("seed", "z", "scope", "root", "clamp_in_split",
                                                          "census_cap", "split", "metric_bounds", "stream",
                                                          "kmeans_k")}
        if kw:
            raise TypeError(f"unknown options {sorted(kw)}")
        tr, dev, keep = _trace(kernel_id, exec_ns, n_kernels, metrics, allow_empty=comm is not None)
        o = _opts(opt.get("seed", 0), opt.get("z", 0.0), opt.get("scope", 0), opt.get("root", True),
                  opt.get("clamp_in_split", True), opt.get("census_cap", False), opt.get("split", 0),
                  opt.get("metric_bounds", False), opt.get("stream"), dev, opt.get("kmeans_k", 3))
        out = C.POINTER(stem_plan)()
        if comm is None:
            st = lib().stem_root_plan_ctx(self._h, C.byref(tr), eps, conf, C.byref(o), C.byref(out))
        else:
            st = lib().stem_root_plan_dist(self._h, comm._h, C.byref(tr), global_row_base, eps, conf, C.byref(o),
                                           C.byref(out))
        _check(st, "stem_root_plan_ctx" if comm is None else "stem_root_plan_dist")
        del keep
        return HostPlan(out)

    def device_plan(self) -> dict:
        v = stem_device_plan()
        _check(lib().stem_ctx_device_plan(self._h, C.byref(v)), "stem_ctx_device_plan")
        return dict(n_clusters=v.n_clusters, n_samples=v.n_samples, clusters=v.clusters, sample_row=v.sample_row,
                    sample_cluster=v.sample_cluster, sample_weight=v.sample_weight, est_total_ns=v.est_total_ns,
                    bound=v.bound, eps=v.eps, z=v.z, true_total_ns=int(v.true_total_ns),
                    est_metric=[v.est_metric[i] for i in range(v.n_metrics)],
                    true_metric=[v.true_metric[i] for i in range(v.n_metrics)] if v.true_metric else None,
                    bound_metric=[v.bound_metric[i] for i in range(v.n_metrics)] if v.bound_metric else None)

    def enable_timing(self, on: bool = True):
        _check(lib().stem_ctx_enable_timing(self._h, int(on)), "stem_ctx_enable_timing")

    def stage_times(self) -> list:
        cnt = C.c_uint32()
        _check(lib().stem_ctx_stage_times(self._h, None, 0, C.byref(cnt)), "stem_ctx_stage_times")
        arr = (stem_stage_time * max(cnt.value, 1))()
        _check(lib().stem_ctx_stage_times(self._h, arr, cnt.value, C.byref(cnt)), "stem_ctx_stage_times")
        return [dict(name=a.name.decode(), ms=a.ms, bytes=a.bytes, launches=a.launches, count=a.count)
                for a in arr[:cnt.value]]

    def stats(self) -> dict:
        s = stem_stats()
        _check(lib().stem_ctx_stats(self._h, C.byref(s)), "stem_ctx_stats")
        return {f: getattr(s, f) for f, _ in stem_stats._fields_}


def plan(kernel_id, exec_ns, n_kernels: int, eps: float = 0.05, conf: float = 0.95, metrics=None, seed: int = 0,
         z: float = 0.0, scope: int = 0, root: bool = True, clamp_in_split: bool = True, census_cap: bool = False,
         stream=None, split: int = 0, metric_bounds: bool = False, kmeans_k: int = 3) -> dict:
    """stem_root_plan: one-shot plan (temporary workspace), host plan out."""
    tr, dev, keep = _trace(kernel_id, exec_ns, n_kernels, metrics)
    o = _opts(seed, z, scope, root, clamp_in_split, census_cap, split, metric_bounds, stream, dev, kmeans_k)
    out = C.POINTER(stem_plan)()
    _check(lib().stem_root_plan(C.byref(tr), eps, conf, C.byref(o), C.byref(out)), "stem_root_plan")
    del keep
    res = _plan_to_numpy(out.contents)
    lib().stem_plan_free(out)
    return res
