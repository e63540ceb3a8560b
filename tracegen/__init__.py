"""Seeded synthetic kernel-invocation traces shaped like the paper's workloads.

This module is the ONE thing the oracle and the CUDA path share: it produces
inputs (kernel_id, exec_ns, metric columns) and holds none of the method's
arithmetic.  Every row is a pure function of (config tables, seed, global row
index), so any shard of rows reproduces the same bytes.

Two implementations of the same per-row recipe:
  * ``generate_np``   -- numpy, the specification (CPU, small sizes);
  * ``generate_cuda`` -- tracegen.cu (libtracegen.so), for bench-size traces
    written straight into HBM.
All transcendental maths (quantile tables, per-kernel parameters) happens
here on the host, once, in numpy fp64; the per-row recipe is integer-only
except the metric columns, which use exactly rounded fp64 mul/add (no FMA), so
the two implementations are byte-identical (tests/test_tracegen.py).

Shapes follow SURVEY.md §8(d) / DESIGN.md §4: kernel frequencies Zipf over a
repeated per-iteration call-site sequence (CASIO/HF traces are iteration loops,
PAPER.md L79-85, Fig. 1), per-kernel execution-time families: narrow unimodal,
multimodal with call-site-tied peaks, wide gamma, heavy-tailed lognormal,
multi-saturation (Fig. 1 L51, Fig. 2; §2).
"""
from __future__ import annotations

import ctypes as C
import dataclasses
import os
import subprocess

import numpy as np

MAXPEAK = 8          # peaks per kernel; peak MAXPEAK-1 is the optional heavy tail
TAB = 4096           # quantile-table resolution (TAB+1 entries per table)
FRAC_BITS = 20       # fixed-point scale of table entries and interpolation
NO_SITE_PEAK = 0xFF  # site_peak value meaning "draw the peak at random"

_HERE = os.path.dirname(os.path.abspath(__file__))


@dataclasses.dataclass
class Spec:
    name: str
    n: int
    n_kernels: int
    seed: int
    eps: float
    conf: float
    site_kid: np.ndarray      # u32 [n_sites]
    site_peak: np.ndarray     # u8  [n_sites]
    pk_cum: np.ndarray        # u32 [K*MAXPEAK] cumulative thresholds for random peaks
    tail_thresh: np.ndarray   # u32 [K] P(tail) * 2^32
    pk_center: np.ndarray     # u32 [K*MAXPEAK] peak centre, ns
    pk_table: np.ndarray      # u16 [K*MAXPEAK] quantile-table index
    tables: np.ndarray        # u32 [n_tables*(TAB+1)] quantile multipliers, 2^-20 fixed point
    n_metrics: int = 0
    mA: np.ndarray = None     # f64 [nm*K]          slope on t
    mB: np.ndarray = None     # f64 [nm*K*MAXPEAK]  per-peak offset
    mS: np.ndarray = None     # f64 [nm*K]          noise scale
    mclamp: np.ndarray = None  # u8 [nm]            1: clamp to [0, 1] (rates, efficiencies)


# ---------------------------------------------------------------- quantile tables
def _norm_ppf(u):
    from scipy.special import ndtri
    return ndtri(u)


def _table(family: str, param: float) -> np.ndarray:
    """Quantile multipliers of a mean-one distribution at u = q/TAB (clipped)."""
    u = np.clip(np.arange(TAB + 1) / TAB, 1e-6, 1 - 1e-6)
    if family == "normal":        # param = CoV
        x = np.maximum(1.0 + param * _norm_ppf(u), 0.02)
    elif family == "lognormal":   # param = sigma of log
        x = np.exp(param * _norm_ppf(u) - 0.5 * param * param)
    elif family == "gamma":       # param = CoV
        from scipy.special import gammaincinv
        k = 1.0 / (param * param)
        x = gammaincinv(k, u) / k
    else:
        raise ValueError(family)
    v = np.round(x * (1 << FRAC_BITS))
    v = np.maximum.accumulate(np.clip(v, 0, 2 ** 32 - 1))
    return v.astype(np.uint32)


class _Tables:
    """Quantised (family, param) -> table index; params snapped to a 1/64 grid."""

    def __init__(self):
        self.keys, self.rows = {}, []

    def get(self, family, param):
        key = (family, round(param * 64) / 64)
        if key not in self.keys:
            self.keys[key] = len(self.rows)
            self.rows.append(_table(*key))
        return self.keys[key]

    def array(self):
        return np.concatenate(self.rows).astype(np.uint32)


# ---------------------------------------------------------------- config builders
def _zipf_sites(rng, K, n_sites, s):
    """Call-site -> kernel map: every kernel once, the rest Zipf(s), shuffled."""
    w = 1.0 / np.arange(1, K + 1) ** s
    rank = rng.permutation(K)                   # which kernel id gets which Zipf rank
    extra = rng.choice(K, n_sites - K, p=w / w.sum())
    sites = np.concatenate([np.arange(K), extra])
    return rank[sites][rng.permutation(n_sites)].astype(np.uint32)


def _build(name, n, K, seed, eps, mix, base_lo_ns, base_hi_ns, n_sites, zipf_s, tail_frac=0.0,
           n_metrics=0, uniform=False, lognormal_sigma=(0.3, 0.8)):
    rng = np.random.default_rng(seed * 1_000_003 + 17)
    tabs = _Tables()
    pk_cum = np.full((K, MAXPEAK), 0xFFFFFFFF, np.uint64)
    pk_center = np.zeros((K, MAXPEAK), np.uint64)
    pk_table = np.zeros((K, MAXPEAK), np.uint16)
    tail = np.zeros(K, np.uint64)
    n_peaks = np.ones(K, np.int64)
    random_peak = np.zeros(K, bool)
    fams = list(mix.keys())
    probs = np.array([mix[f] for f in fams])
    kind = rng.choice(len(fams), K, p=probs / probs.sum())
    base = np.exp(rng.uniform(np.log(base_lo_ns), np.log(base_hi_ns), K))
    for k in range(K):
        f = fams[kind[k]]
        if f == "narrow":                       # sgemm-like: CoV 0.5-5 %
            pk_center[k, 0] = base[k]
            pk_table[k, 0] = tabs.get("normal", rng.uniform(0.005, 0.05))
        elif f == "bimodal":                    # C1: two Gaussians, sigma 2 %, random weight
            mu2 = base[k] * rng.uniform(1.5, 3.0)
            pk_center[k, :2] = [base[k], mu2]
            pk_table[k, :2] = tabs.get("normal", 0.02)
            w = rng.uniform(0.2, 0.8)
            pk_cum[k, 0] = int(w * 2 ** 32)
            n_peaks[k], random_peak[k] = 2, True
        elif f == "multimodal":                 # bn_fw_inf-like: 2-4 peaks 1.2-3x apart
            p = rng.integers(2, 5)
            ratios = np.cumprod(np.concatenate([[1.0], rng.uniform(1.2, 3.0, p - 1)]))
            pk_center[k, :p] = base[k] * ratios
            for j in range(p):
                pk_table[k, j] = tabs.get("normal", rng.uniform(0.01, 0.04))
            n_peaks[k] = p
        elif f == "multisat":                   # LLM multi-saturation: 3-6 narrow peaks
            p = rng.integers(3, 7)
            ratios = np.cumprod(np.concatenate([[1.0], rng.uniform(1.15, 2.0, p - 1)]))
            pk_center[k, :p] = base[k] * ratios
            for j in range(p):
                pk_table[k, j] = tabs.get("normal", rng.uniform(0.003, 0.02))
            n_peaks[k] = p
        elif f == "gamma":                      # max_pool-like: wide, CoV 20-60 %
            pk_center[k, 0] = base[k]
            pk_table[k, 0] = tabs.get("gamma", rng.uniform(0.2, 0.6))
        elif f == "lognormal":                  # heavy tail
            lo, hi = lognormal_sigma
            pk_center[k, 0] = base[k]
            pk_table[k, 0] = tabs.get("lognormal", rng.uniform(lo, hi))
        if tail_frac and rng.random() < 0.3:    # training-shaped lognormal tail
            pk_center[k, MAXPEAK - 1] = base[k] * 1.5
            pk_table[k, MAXPEAK - 1] = tabs.get("lognormal", 1.0)
            tail[k] = int(tail_frac * 2 ** 32)
    if uniform:
        site_kid = np.arange(K, dtype=np.uint32)
    else:
        site_kid = _zipf_sites(rng, K, n_sites, zipf_s)
    site_peak = np.zeros(len(site_kid), np.uint8)
    for s in range(len(site_kid)):
        k = site_kid[s]
        site_peak[s] = NO_SITE_PEAK if random_peak[k] else rng.integers(0, n_peaks[k])
    # a peak's time must stay below 2^32 ns after the largest multiplier
    pk_center = np.minimum(pk_center, 2 ** 27).astype(np.uint32)
    spec = Spec(name, n, K, seed, eps, 0.95, site_kid, site_peak,
                pk_cum.astype(np.uint32).ravel(), tail.astype(np.uint32), pk_center.ravel(),
                pk_table.ravel(), tabs.array())
    if n_metrics:
        nm = n_metrics
        spec.n_metrics = nm
        # per-kernel linear maps of t + per-peak offsets + noise:
        # counts (instructions, transactions), rates in [0,1] (hit rates), efficiencies
        clamp = np.array([0, 0, 0, 0, 1, 1, 1, 1, 0, 0, 1, 1][:nm] + [0] * max(0, nm - 12), np.uint8)
        A = np.where(clamp[:, None] == 1, rng.uniform(0, 1e-7, (nm, K)), rng.uniform(0.5, 40.0, (nm, K)))
        B = np.where(clamp[:, None, None] == 1, rng.uniform(0.2, 0.9, (nm, K, MAXPEAK)),
                     rng.uniform(0, 5e4, (nm, K, MAXPEAK)))
        S = np.where(clamp[:, None] == 1, rng.uniform(0.0, 0.1, (nm, K)), rng.uniform(0, 1e3, (nm, K)))
        spec.mA, spec.mB, spec.mS, spec.mclamp = A.ravel(), B.ravel(), S.ravel(), clamp
    return spec


CONFIGS = {
    # SURVEY.md §8(d) / BASELINE.json configs[0..4]
    "C1": lambda n=10_000, seed=1: _build("C1", n, 20, seed, 0.05, {"bimodal": 1.0}, 2e3, 50e3, 20, 0.0,
                                          uniform=True),
    "C2": lambda n=1_000_000, seed=2: _build("C2", n, 500, seed, 0.05,
                                             {"narrow": .40, "multimodal": .25, "gamma": .20, "lognormal": .15},
                                             2e3, 2e6, 8192, 1.1),
    "C3": lambda n=20_000_000, seed=3: _build("C3", n, 2000, seed, 0.05,
                                              {"lognormal": .50, "multisat": .30, "narrow": .20},
                                              2e3, 4e6, 32768, 1.1, n_metrics=12, lognormal_sigma=(0.5, 1.2)),
    "C4": lambda n=100_000_000, seed=4: _build("C4", n, 1000, seed, 0.05,
                                               {"narrow": .40, "multimodal": .25, "gamma": .20, "lognormal": .15},
                                               2e3, 2e6, 16384, 1.1, tail_frac=0.02),
    "C5": lambda n=1_000_000_000, seed=5: _build("C5", n, 10_000, seed, 0.05,
                                                 {"lognormal": .50, "multisat": .30, "narrow": .20},
                                                 2e3, 4e6, 65536, 1.1, lognormal_sigma=(0.5, 1.2)),
}


def spec(name: str, n: int | None = None, seed: int | None = None) -> Spec:
    kw = {}
    if n is not None:
        kw["n"] = n
    if seed is not None:
        kw["seed"] = seed
    return CONFIGS[name](**kw)


# ---------------------------------------------------------------- per-row recipe (numpy spec)
_M64 = np.uint64(0xFFFFFFFFFFFFFFFF)


def _splitmix(x):
    with np.errstate(over="ignore"):
        x = x + np.uint64(0x9E3779B97F4A7C15)
        x = (x ^ (x >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
        x = (x ^ (x >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
        return x ^ (x >> np.uint64(31))


def _hash(seed, rows, stream):
    with np.errstate(over="ignore"):
        x = np.uint64(seed) ^ (rows * np.uint64(0xD1B54A32D192ED03)) ^ np.uint64((stream * 0x8CB92BA72F3D8DD7)
                                                                               & 0xFFFFFFFFFFFFFFFF)
    return _splitmix(x)


def generate_np(sp: Spec, row0: int = 0, count: int | None = None):
    """Rows [row0, row0+count) of the trace.  Returns (kid u32, t u32, metrics f64 [nm, count] | None)."""
    count = sp.n - row0 if count is None else count
    r = np.arange(row0, row0 + count, dtype=np.uint64)
    site = (r % np.uint64(len(sp.site_kid))).astype(np.int64)
    kid = sp.site_kid[site].astype(np.int64)
    h1 = _hash(sp.seed, r, 1)
    u_hi = (h1 >> np.uint64(32)).astype(np.uint64)
    u_lo = (h1 & np.uint64(0xFFFFFFFF)).astype(np.uint64)
    peak = sp.site_peak[site].astype(np.int64)
    rnd = peak == NO_SITE_PEAK
    if rnd.any():
        cum = sp.pk_cum.reshape(-1, MAXPEAK)[kid[rnd]].astype(np.uint64)
        p = np.zeros(rnd.sum(), np.int64)
        for j in range(MAXPEAK - 1):
            p += (p == j) & (u_hi[rnd] >= cum[:, j])
        peak[rnd] = p
    is_tail = u_lo < sp.tail_thresh[kid].astype(np.uint64)
    peak[is_tail] = MAXPEAK - 1
    idx = kid * MAXPEAK + peak
    h2 = _hash(sp.seed, r, 2)
    q = (h2 >> np.uint64(52)).astype(np.int64)
    frac = (h2 >> np.uint64(32)) & np.uint64((1 << FRAC_BITS) - 1)
    tb = sp.pk_table[idx].astype(np.int64) * (TAB + 1) + q
    a = sp.tables[tb].astype(np.uint64)
    b = sp.tables[tb + 1].astype(np.uint64)
    v = a + (((b - a) * frac) >> np.uint64(FRAC_BITS))
    t = (sp.pk_center[idx].astype(np.uint64) * v) >> np.uint64(FRAC_BITS)
    t = np.minimum(t, np.uint64(0xFFFFFFFF)).astype(np.uint32)
    met = None
    if sp.n_metrics:
        K = sp.n_kernels
        tf = t.astype(np.float64)
        met = np.empty((sp.n_metrics, count), np.float64)
        for c in range(sp.n_metrics):
            u = (_hash(sp.seed, r, 3 + c) >> np.uint64(11)).astype(np.float64) * 2.0 ** -53
            x = sp.mA[c * K + kid] * tf
            y = sp.mS[c * K + kid] * u
            z = sp.mB[(c * K + kid) * MAXPEAK + peak] + y
            val = x + z
            if sp.mclamp[c]:
                val = np.minimum(np.maximum(val, 0.0), 1.0)
            met[c] = val
    return kid.astype(np.uint32), t, met


# ---------------------------------------------------------------- CUDA twin
_LIB = os.path.join(_HERE, "libtracegen.so")
_SRC = os.path.join(_HERE, "tracegen.cu")
_lib = None


def build(force=False):
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        subprocess.check_call(["nvcc", "-O3", "-gencode", "arch=compute_100a,code=sm_100a", "-lineinfo",
                               "--fmad=false", "-Xcompiler", "-fPIC", "-shared", "-o", _LIB, _SRC])
    return _LIB


def _cuda_lib():
    global _lib
    if _lib is None:
        _lib = C.CDLL(build())
        _lib.tg_generate.restype = C.c_int
        _lib.tg_generate.argtypes = [C.c_uint64, C.c_uint64, C.c_uint64, C.c_uint32] + [C.c_void_p] * 7 + \
            [C.c_uint32, C.c_uint32] + [C.c_void_p] * 4 + [C.c_void_p] * 3 + [C.c_uint64, C.c_void_p]
    return _lib


class DeviceSpec:
    """Spec tables resident on a CUDA device (torch tensors)."""

    def __init__(self, sp: Spec, device):
        import torch

        def dev(a, dt=None):
            return torch.from_numpy(np.ascontiguousarray(a if dt is None else a.astype(dt))).to(device)
        self.sp = sp
        self.site_kid = dev(sp.site_kid.view(np.int32))
        self.site_peak = dev(sp.site_peak)
        self.pk_cum = dev(sp.pk_cum.view(np.int32))
        self.tail = dev(sp.tail_thresh.view(np.int32))
        self.center = dev(sp.pk_center.view(np.int32))
        self.ptab = dev(sp.pk_table.view(np.int16))
        self.tables = dev(sp.tables.view(np.int32))
        if sp.n_metrics:
            self.mA, self.mB, self.mS = dev(sp.mA), dev(sp.mB), dev(sp.mS)
            self.mclamp = dev(sp.mclamp)


def generate_cuda(ds: DeviceSpec, kid_out, t_out, met_out=None, row0=0, count=None, stream=None):
    """Write rows [row0, row0+count) into device tensors (int32 views of u32; met [nm, count] f64)."""
    import torch
    sp = ds.sp
    count = kid_out.numel() if count is None else count
    st = torch.cuda.current_stream().cuda_stream if stream is None else stream
    nm = sp.n_metrics if met_out is not None else 0
    ptr = lambda x: None if x is None else x.data_ptr()  # noqa: E731
    rc = _cuda_lib().tg_generate(
        sp.seed, row0, count, len(sp.site_kid),
        ptr(ds.site_kid), ptr(ds.site_peak), ptr(ds.pk_cum), ptr(ds.tail), ptr(ds.center), ptr(ds.ptab),
        ptr(ds.tables), sp.n_kernels, nm,
        ptr(ds.mA) if nm else None, ptr(ds.mB) if nm else None, ptr(ds.mS) if nm else None,
        ptr(ds.mclamp) if nm else None,
        ptr(kid_out), ptr(t_out), ptr(met_out) if nm else None, count, st)
    if rc != 0:
        raise RuntimeError(f"tg_generate failed: {rc}")
