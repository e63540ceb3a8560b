#include <cstdio>
// root.cu -- steps a2-a4: sampled exact prefix moments of the grouped times
// and the level-synchronous ROOT clustering (§3.4, Fig. 6).
//
// Every level processes the whole frontier (all kernels' active clusters at
// once).  For each cluster the 2-means cut (R5) is the argmax over its cuts k
// of D_k^2/(k(n-k)), D_k = n S_L(k) - S k, compared exactly:
//   local_root_kernel   clusters < big_rows(): one warp finishes the cluster's
//                       whole ROOT subtree (cut, Eq. 7/8 decision, children)
//                       depth first, rows re-read from L1/L2 instead of one
//                       frontier pass per level
//   big_split_kernel    clusters >= big_rows(): one block per 65536 rows,
//                       chunk bounds from the sampled prefix, only chunks that
//                       may hold the argmax are scanned; big_reduce_kernel
//   decide_kernel       Eq. 7 vs Eq. 8 per big cluster (R6-R9), fixed fp64 order
//   scan + apply        compacts the non-trivial children into the next frontier
// The decision of a cluster depends on its rows alone, so the order in which
// clusters are finished does not change the leaves (flags at the cut rows).
// Cluster totals (S exact u64, Q exact u128) travel with the frontier; only
// Q_L at the chosen cut is read from the sampled prefix arrays.
#include <cstdlib>

#include "internal.h"

namespace sr {

// clusters of >= big_rows() rows take the chunk-bound path (STEMROOT_BIG_ROWS overrides)
__constant__ uint64_t c_big;
__constant__ int c_bound2;   // 1: two-sided chunk bounds on the big path (STEMROOT_SPLIT_BOUND=1)
static uint64_t big_rows() {
    static uint64_t v = 0;
    if (!v) {
        const char *e = getenv("STEMROOT_BIG_ROWS");
        v = e ? strtoull(e, nullptr, 10) : 2048;
        if (v < 64) v = 64;
    }
    return v;
}
#ifndef SR_BIG_SEG
#define SR_BIG_SEG 65536
#endif
constexpr uint64_t kBigSeg = SR_BIG_SEG;               // rows per block on the big-cluster path
// clusters of < local_rows() rows are finished by local_root_kernel
// (STEMROOT_LOCAL_ROWS, default 0 = off: measured slower than the level loop
// on C5)
__constant__ uint64_t c_loc;
static bool split_overlap() {   // STEMROOT_SPLIT_OVERLAP=0: small and big split in sequence
    static int v = -1;
    if (v < 0) v = (getenv("STEMROOT_SPLIT_OVERLAP") && getenv("STEMROOT_SPLIT_OVERLAP")[0] == '0') ? 0 : 1;
    return v == 1;
}
// exact split rule's kernels: 2 (default) the nearest-centre descent for every
// cluster; 1 the descent for big clusters, chunk bounds for the small ones; 0
// chunk bounds for all (small-cluster warps + big-cluster blocks, the round-1/2
// design).  STEMROOT_SPLIT_NC, read per plan.  C5: root_split 6.5 ms (0), 3.6 (1), 2.2 (2).
static int nc_mode() {
    const char *e = getenv("STEMROOT_SPLIT_NC");
    return e ? atoi(e) : 2;
}
static bool seed_on() {   // STEMROOT_SPLIT_SEED=0 disables the coarse threshold seed
    static int v = -1;
    if (v < 0) v = (getenv("STEMROOT_SPLIT_SEED") && getenv("STEMROOT_SPLIT_SEED")[0] == '0') ? 0 : 1;
    return v == 1;
}
static bool debug_levels() {
    static int v = -1;
    if (v < 0) v = getenv("STEMROOT_DEBUG_LEVELS") ? 1 : 0;
    return v == 1;
}
static uint64_t local_rows() {
    static uint64_t v = ~0ull;
    if (v == ~0ull) {
        const char *e = getenv("STEMROOT_LOCAL_ROWS");
        v = e ? strtoull(e, nullptr, 10) : 0;
    }
    return v;
}

struct SQ {
    uint64_t s;
    u128 q;
};
__host__ __device__ __forceinline__ SQ operator+(const SQ &a, const SQ &b) { return SQ{a.s + b.s, a.q + b.q}; }
__host__ __device__ __forceinline__ SQ operator-(const SQ &a, const SQ &b) { return SQ{a.s - b.s, a.q - b.q}; }

// ---------------------------------------------------------------- a2: sampled P1, P2
// Three launches, each a coalesced stream (no look-back chain: a single-pass
// decoupled look-back was measured slower, its tiles waiting on predecessors):
//  1. pm_sums: a block per tile of kPmChunks 32-row chunks sums t and t^2 per
//     chunk (eight lanes per chunk, one uint4 each, eight warp loads in
//     flight), writes the chunk sums, the tile total and the chunk-boundary
//     pairs TB[j] = (t[32 j - 1], t[32 j]) that the split bounds read;
//  2. pm_tiles: one block scans the tile totals;
//  3. pm_apply: a block per tile scans its chunk sums and writes PS1/PS2.
// Element j of the scan is chunk j (zero for j >= nchunks), j in [0, nchunks].
// Bytes: 4 per row + 24 + 24 + 24 (+ 8 TB) per chunk.
constexpr int kPmThreads = 256, kPmChunks = 2 * kPmThreads;   // 16 384 rows per tile
constexpr int kPmScanBlock = 1024;                                // tile totals per pm_tiles block
struct SQ3 {   // chunk sums, 24 B
    uint64_t s, lo, hi;
};

__device__ __forceinline__ void add128(uint64_t &lo, uint64_t &hi, uint64_t ol, uint64_t oh) {
    const uint64_t nl = lo + ol;
    hi += oh + (nl < lo);
    lo = nl;
}

__global__ void __launch_bounds__(kPmThreads) pm_sums_kernel(const uint32_t *__restrict__ t, uint64_t n,
                                                             uint64_t nchunks, SQ3 *__restrict__ csum,
                                                             SQ *__restrict__ tile_tot, uint32_t *__restrict__ TB) {
    __shared__ SQ s_part[kPmThreads / 32];
    const int tid = threadIdx.x, lane = tid & 31, sub = lane & 3, grp = lane >> 2, w = tid >> 5;
    const uint64_t c0 = (uint64_t)blockIdx.x * kPmChunks;
    const bool vec = (reinterpret_cast<uintptr_t>(t) & 15) == 0;
    // four lanes per chunk, two uint4 each (lane sub covers rows 8 sub .. 8 sub + 7
    // of the chunk); eight chunks per warp step; kU steps of loads in flight
    constexpr int kPerWarp = kPmChunks / (kPmThreads / 32), kU = 4;   // 64 chunks per warp
    uint64_t as = 0, al = 0, ah = 0;
#pragma unroll
    for (int r = 0; r < kPerWarp / (8 * kU); r++) {
        uint4 v[kU][2];
#pragma unroll
        for (int u = 0; u < kU; u++) {
            const uint64_t j = c0 + w * kPerWarp + (r * kU + u) * 8 + grp;
            const uint64_t i = j * kChunk + sub * 8;
#pragma unroll
            for (int h = 0; h < 2; h++) {
                const uint64_t ih = i + 4 * h;
                if (vec && ih + 3 < n) {
                    v[u][h] = __ldcs(reinterpret_cast<const uint4 *>(t + ih));
                } else {
                    v[u][h].x = ih < n ? t[ih] : 0;
                    v[u][h].y = ih + 1 < n ? t[ih + 1] : 0;
                    v[u][h].z = ih + 2 < n ? t[ih + 2] : 0;
                    v[u][h].w = ih + 3 < n ? t[ih + 3] : 0;
                }
            }
        }
#pragma unroll
        for (int u = 0; u < kU; u++) {
            uint64_t s = 0, qlo = 0, qhi = 0;
#pragma unroll
            for (int h = 0; h < 2; h++) {
                const uint64_t x0 = v[u][h].x, x1 = v[u][h].y, x2 = v[u][h].z, x3 = v[u][h].w;
                s += x0 + x1 + x2 + x3;
                const uint64_t a0 = x0 * x0, a1 = x1 * x1, a2 = x2 * x2, a3 = x3 * x3;
                add128(qlo, qhi, a0, 0);
                add128(qlo, qhi, a1, 0);
                add128(qlo, qhi, a2, 0);
                add128(qlo, qhi, a3, 0);
            }
#pragma unroll
            for (int o = 2; o; o >>= 1) {
                s += __shfl_xor_sync(0xffffffffu, s, o);
                const uint64_t ol = __shfl_xor_sync(0xffffffffu, qlo, o), oh = __shfl_xor_sync(0xffffffffu, qhi, o);
                add128(qlo, qhi, ol, oh);
            }
            const uint64_t j = c0 + w * kPerWarp + (r * kU + u) * 8 + grp;
            if (sub == 0) {
                as += s;
                add128(al, ah, qlo, qhi);
                if (j <= nchunks) csum[j] = SQ3{s, qlo, qhi};
                if (j < nchunks) {
                    TB[2 * j + 1] = v[u][0].x;                 // t[32 j]
                    if (j == 0) TB[0] = 0;
                }
            }
            if (sub == 3 && j + 1 < nchunks) TB[2 * (j + 1)] = v[u][1].w;   // t[32 (j + 1) - 1]
        }
    }
    // tile total (lanes sub != 0 hold zero)
#pragma unroll
    for (int o = 16; o; o >>= 1) {
        as += __shfl_xor_sync(0xffffffffu, as, o);
        const uint64_t ol = __shfl_xor_sync(0xffffffffu, al, o), oh = __shfl_xor_sync(0xffffffffu, ah, o);
        add128(al, ah, ol, oh);
    }
    if (lane == 0) s_part[w] = SQ{as, ((u128)ah << 64) | al};
    __syncthreads();
    if (tid == 0) {
        SQ tot{0, 0};
        for (int k = 0; k < kPmThreads / 32; k++) tot = tot + s_part[k];
        tile_tot[blockIdx.x] = tot;
    }
}

// a block per kPmScanBlock tile totals: exclusive scan in place, the block's
// total to btot[blockIdx]
__global__ void __launch_bounds__(kPmScanBlock) pm_tiles_kernel(SQ *__restrict__ tile_tot, uint64_t ntiles,
                                                                SQ *__restrict__ btot) {
    __shared__ SQ sm[kPmScanBlock / 32 + 1];
    const uint64_t i = (uint64_t)blockIdx.x * kPmScanBlock + threadIdx.x;
    const SQ v = i < ntiles ? tile_tot[i] : SQ{0, 0};
    SQ tot;
    const SQ ex = block_excl_scan<SQ, kPmScanBlock>(v, sm, &tot);
    if (i < ntiles) tile_tot[i] = ex;
    if (threadIdx.x == 0) btot[blockIdx.x] = tot;
}

__global__ void __launch_bounds__(kPmThreads) pm_apply_kernel(const SQ3 *__restrict__ csum, uint64_t nchunks,
                                                              const SQ *__restrict__ tile_pre, const SQ *__restrict__ btot,
                                                              uint64_t ntiles, uint64_t *__restrict__ PS1,
                                                              u128 *__restrict__ PS2, uint64_t *__restrict__ total) {
    __shared__ SQ s_scan[kPmThreads / 32 + 1];
    __shared__ SQ s_base;
    const int tid = threadIdx.x, lane = tid & 31;
    if (tid < 32) {   // sum of the pm_tiles blocks before this tile's
        const uint32_t nb = blockIdx.x / kPmScanBlock;
        uint64_t bs = 0, bl = 0, bh = 0;
        for (uint32_t k = lane; k < nb; k += 32) {
            const SQ x = btot[k];
            bs += x.s;
            add128(bl, bh, (uint64_t)x.q, (uint64_t)(x.q >> 64));
        }
#pragma unroll
        for (int o = 16; o; o >>= 1) {
            bs += __shfl_xor_sync(0xffffffffu, bs, o);
            const uint64_t ol = __shfl_xor_sync(0xffffffffu, bl, o), oh = __shfl_xor_sync(0xffffffffu, bh, o);
            add128(bl, bh, ol, oh);
        }
        if (lane == 0) s_base = SQ{bs, ((u128)bh << 64) | bl} + tile_pre[blockIdx.x];
    }
    const uint64_t j0 = (uint64_t)blockIdx.x * kPmChunks + 2 * tid;
    SQ e0{0, 0}, e1{0, 0};
    if (j0 <= nchunks) { const SQ3 x = csum[j0]; e0 = SQ{x.s, ((u128)x.hi << 64) | x.lo}; }
    if (j0 + 1 <= nchunks) { const SQ3 x = csum[j0 + 1]; e1 = SQ{x.s, ((u128)x.hi << 64) | x.lo}; }
    SQ tot;
    const SQ ex = block_excl_scan<SQ, kPmThreads>(e0 + e1, s_scan, &tot);   // (syncs: s_base visible)
    const SQ p0 = s_base + ex, p1 = p0 + e0;
    if (j0 + 1 <= nchunks) {
        reinterpret_cast<ulonglong2 *>(PS1)[j0 >> 1] = make_ulonglong2(p0.s, p1.s);
        PS2[j0] = p0.q;
        PS2[j0 + 1] = p1.q;
    } else if (j0 <= nchunks) {
        PS1[j0] = p0.s;
        PS2[j0] = p0.q;
    }
    if (tid == 0 && blockIdx.x + 1 == ntiles) {   // the tile holding element nchunks: grand total
        const SQ g = s_base + tot;
        total[0] = g.s;
        total[1] = (uint64_t)g.q;
        total[2] = (uint64_t)(g.q >> 64);
    }
}

int prefix_moments(Ctx &c, uint64_t n) {
    const uint64_t nchunks = (n + kChunk - 1) / kChunk;
    const uint64_t ntiles = (nchunks + 1 + kPmChunks - 1) / kPmChunks;
    const uint64_t nblk = (ntiles + kPmScanBlock - 1) / kPmScanBlock;
    CKS(c.ensure(c.chunk_sq, c.cap_chunk_sq, sizeof(SQ3) * (ntiles * kPmChunks) + sizeof(SQ) * (ntiles + nblk + 1)));
    CKS(c.ensure(c.TB, c.cap_TB, sizeof(uint32_t) * 2 * (nchunks + 1)));
    SQ3 *csum = (SQ3 *)c.chunk_sq;
    SQ *ttot = (SQ *)(csum + ntiles * kPmChunks), *btot = ttot + ntiles;
    const int tk = c.stage_begin("prefix_moments");
    pm_sums_kernel<<<(unsigned)ntiles, kPmThreads, 0, c.stream>>>(c.t_sorted, n, nchunks, csum, ttot, c.TB);
    pm_tiles_kernel<<<(unsigned)nblk, kPmScanBlock, 0, c.stream>>>(ttot, ntiles, btot);
    pm_apply_kernel<<<(unsigned)ntiles, kPmThreads, 0, c.stream>>>(csum, nchunks, ttot, btot, ntiles, c.PS1, c.PS2,
                                                                   c.scalars->wide_total);
    c.launches += 3;
    c.stage_end(tk, 4 * n + 24 * (nchunks + 1));
    CK(cudaGetLastError());
    return STEM_OK;
}

// ---------------------------------------------------------------- a3: split
__device__ __forceinline__ bool nontrivial(const uint32_t *t, uint32_t lo, uint32_t hi) {
    return hi - lo >= 2 && t[lo] != t[hi - 1];
}

// Evaluate the valid cut k (t[k-1] < t[k]): |D| = S k - n S_L (D <= 0 for sorted
// data) computed exactly here, only at distinct-value boundaries.
__device__ __forceinline__ void eval_cut(uint32_t k, uint64_t n, uint64_t S, uint64_t SL, Cand &best) {
    const u128 ad = (u128)S * k - (u128)n * SL;
    const uint32_t dhi = (uint32_t)(ad >> 64);
    const uint64_t dlo = (uint64_t)ad;
    const double dD = approx_d(dhi, dlo);
    const double x = __dmul_rn(dD, dD);
    const double dp = __dmul_rn(__uint2double_rn(k), __uint2double_rn((uint32_t)(n - k)));
    bool take = best.k == 0;
    if (!take) {
        const double L = __dmul_rn(x, best.dp), R = __dmul_rn(best.x, dp);
        const double tol = 1.0 + 0x1p-40;
        if (L > __dmul_rn(R, tol)) {
            take = true;
        } else if (!(R > __dmul_rn(L, tol))) {            // near tie: exact 256-bit products
            Cand cd;
            cd.dlo = dlo;
            cd.dhi = dhi;
            cd.p = (uint64_t)k * (n - k);
            const int cmp = exact_cmp(cd, best);          // equal -> the smaller k (any scan order)
            take = cmp > 0 || (cmp == 0 && k < best.k);
        }
    }
    if (take) {
        best.x = x;
        best.dp = dp;
        best.dlo = dlo;
        best.dhi = dhi;
        best.p = (uint64_t)k * (n - k);
        best.SL = SL;
        best.k = k;
    }
}

__device__ __forceinline__ Cand shfl_cand_xor(const Cand &a, int m) {
    Cand r;
    r.x = __shfl_xor_sync(0xffffffffu, a.x, m);
    r.dp = __shfl_xor_sync(0xffffffffu, a.dp, m);
    r.dlo = __shfl_xor_sync(0xffffffffu, a.dlo, m);
    r.p = __shfl_xor_sync(0xffffffffu, a.p, m);
    r.SL = __shfl_xor_sync(0xffffffffu, a.SL, m);
    r.dhi = __shfl_xor_sync(0xffffffffu, a.dhi, m);
    r.k = __shfl_xor_sync(0xffffffffu, a.k, m);
    return r;
}

// ---------------------------------------------------------------- warp argmax over one cluster
// Best valid cut of t[lo, lo + n) (S = its sum), 32 rows per step: coalesced
// loads, a warp scan gives S_L, every valid cut is scored exactly (eval_cut).
// A 32-row chunk is skipped when the concavity bound of its cuts is below the
// best candidate so far (exact-safe, see big_split_kernel).  Every lane
// returns the same candidate.
__device__ __forceinline__ Cand warp_scan_cut(const uint32_t *__restrict__ t, uint64_t lo, uint64_t n, uint64_t S) {
    constexpr int kQ = 2;   // 32-row chunks loaded per step
    const int lane = threadIdx.x & 31;
    const double up = 1.0 + 0x1p-44, dn = 1.0 - 0x1p-44;
    Cand best = no_cand();
    double thr = 0.0;
    uint64_t SLb = 0;
    uint32_t tlast = 0;
    for (uint64_t kb = 0; kb < n; kb += 32 * kQ) {
        uint32_t tq[kQ];
#pragma unroll
        for (int q = 0; q < kQ; q++) {
            const uint64_t k = kb + 32 * q + lane;
            tq[q] = k < n ? t[lo + k] : 0u;
        }
#pragma unroll
        for (int q = 0; q < kQ; q++) {
            const uint64_t k0 = kb + 32 * q;
            if (k0 >= n) break;
            const uint64_t k = k0 + lane;
            const bool in = k < n;
            const uint32_t tc = tq[q];
            uint32_t tp = __shfl_up_sync(0xffffffffu, tc, 1);
            if (lane == 0) tp = tlast;
            uint64_t incl = tc;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const uint64_t v = __shfl_up_sync(0xffffffffu, incl, o);
                if (lane >= o) incl += v;
            }
            // upper bound of the chunk's scores from its first cut (warp-uniform)
            const uint64_t cnt = min((uint64_t)32, n - k0);
            const uint32_t t0 = __shfl_sync(0xffffffffu, tc, 0);
            const u128 ad0 = (u128)S * k0 - (u128)n * SLb;
            const uint64_t nt0 = n * (uint64_t)t0;
            const double slope = S > nt0 ? __ull2double_rn(S - nt0) : 0.0;
            const double dub = __dmul_rn(__dadd_rn(approx_d((uint32_t)(ad0 >> 64), (uint64_t)ad0),
                                                   __dmul_rn(slope, (double)(cnt - 1))), up);
            const uint64_t kf = max(k0, (uint64_t)1), kl = min(k0 + cnt - 1, n - 1);
            double ub = 0.0;
            if (kf <= kl) {
                const double pmin =
                    fmin(__dmul_rn((double)kf, (double)(n - kf)), __dmul_rn((double)kl, (double)(n - kl)));
                ub = __dmul_rn(__ddiv_rn(__dmul_rn(dub, dub), pmin), up);
            }
            if (ub >= thr) {
                if (in && k >= 1 && tp < tc) eval_cut((uint32_t)k, n, S, SLb + incl - tc, best);
                double lb = best.k ? __dmul_rn(__ddiv_rn(best.x, best.dp), dn) : 0.0;
#pragma unroll
                for (int o = 16; o; o >>= 1) lb = fmax(lb, __shfl_xor_sync(0xffffffffu, lb, o));
                thr = fmax(thr, lb);
            }
            SLb += __shfl_sync(0xffffffffu, incl, 31);
            tlast = __shfl_sync(0xffffffffu, tc, 31);
        }
    }
#pragma unroll 1   // one copy of better() (with its 256-bit tie path) in the kernel body
    for (int o = 16; o; o >>= 1) {
        const Cand v = shfl_cand_xor(best, o);
        if (better(v, best)) best = v;
    }
    return best;
}

// lower bound of x / p (x, p > 0): fast reciprocal refined by one Newton step,
// scaled down by 2^-30 to cover its error (a smaller lower bound only prunes less)
__device__ __forceinline__ double div_lower(double x, double p) {
    double r;
    asm("rcp.approx.ftz.f64 %0, %1;" : "=d"(r) : "d"(p));
    r = __fma_rn(r, __fma_rn(-p, r, 1.0), r);
    return __dmul_rn(__dmul_rn(x, r), 1.0 - 0x1p-30);
}

// upper bound of x / p (x >= 0, p > 0): as div_lower, scaled up by 2^-30
__device__ __forceinline__ double div_upper(double x, double p) {
    double r;
    asm("rcp.approx.ftz.f64 %0, %1;" : "=d"(r) : "d"(p));
    r = __fma_rn(r, __fma_rn(-p, r, 1.0), r);
    return __dmul_rn(__dmul_rn(x, r), 1.0 + 0x1p-30);
}

// Upper bound of ad_k = S k - n S_L(k) (>= 0 for sorted rows) over the cuts
// k in [ka, ka + cnt - 1] of one chunk, from A = ad_ka and the chunk's first
// time ta.  ad is concave in k (its increments S - n t_j fall as t rises), so it
// lies below the tangent at the chunk start (slope S - n ta) and, when the
// exact E = ad at ka + cnt and the chunk's last time tl are known (has_e),
// below the line through that point with slope S - n tl: the bound is the
// value where the two lines cross.  fp64 with the roundings covered: every
// term is nonnegative and within a few ulps of max(A, E), the crossing uses an
// upward-rounded division, and the result gets 2^-46 max(A, E) of absolute
// slack (the callers also scale it up).
__device__ __forceinline__ double chunk_ad_bound(double A, uint64_t n, uint64_t S, uint32_t ta, uint64_t cnt,
                                                 bool has_e, double E, uint32_t tl) {
    const uint64_t nta = n * (uint64_t)ta;
    if (S <= nta) return A;                                 // increments <= 0: the maximum is at ka
    const double sa = __ull2double_rn(S - nta);
    const double U1 = __dadd_rn(A, __dmul_rn(sa, (double)(cnt - 1)));   // tangent at the start
    if (!has_e) return U1;
    const double slack = __dmul_rn(fmax(A, E), 0x1p-46);
    const uint64_t ntl = n * (uint64_t)tl;
    if (S >= ntl) return fmin(U1, __dadd_rn(E, slack));      // increments >= 0: ad <= ad at ka + cnt
    const double sb = __ull2double_rn(ntl - S);               // |last increment|
    // A + sa x = E + sb (cnt - x) at x = (E - A + sb cnt) / (sa + sb)
    const double num = __dadd_rn(__dsub_rn(E, A), __dmul_rn(sb, (double)cnt));
    const double x = num > 0.0 ? div_upper(num, __dadd_rn(sa, sb)) : 0.0;
    const double Uc = __dadd_rn(__dadd_rn(A, __dmul_rn(sa, x)), slack);
    return fmin(U1, Uc);
}

// Warp scan of the rows [ra, rb) of a cluster starting at lo (S_L at ra = SLa):
// every valid cut is scored exactly into best.
__device__ __forceinline__ void scan_chunk(const uint32_t *__restrict__ t, uint64_t lo, uint64_t n, uint64_t S,
                                           uint64_t ra, uint64_t rb, uint64_t SLa, Cand &best) {
    const int lane = threadIdx.x & 31;
    SR_DCHECK(ra >= lo && rb <= lo + n && rb - ra <= 32);
    const uint64_t row = ra + lane;
    const bool in = row < rb;
    const uint32_t tc = in ? t[row] : 0u;
    uint32_t tp = __shfl_up_sync(0xffffffffu, tc, 1);
    if (lane == 0) tp = row > lo ? t[row - 1] : 0u;
    uint64_t incl = tc;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const uint64_t v = __shfl_up_sync(0xffffffffu, incl, o);
        if (lane >= o) incl += v;
    }
    const uint64_t k = row - lo;
    if (in && k >= 1 && tp < tc) eval_cut((uint32_t)k, n, S, SLa + incl - tc, best);
}

// Best valid cut k with lo + k in [r0, r1) of the cluster [lo, lo + n) (sum S,
// base = sum of t before lo), by chunk bounds: the rows are cut into 32-row
// chunks aligned to the sampled prefix; lane i bounds chunk i from S_L at its
// start (PS1, exact) and t there (TB), and scores the chunk start when it is a
// valid cut (a real candidate: a lower bound of the argmax).  Only chunks
// whose bound reaches the best lower bound are scanned row by row, and every
// scored candidate raises that threshold.  With cthr != NULL the threshold is
// shared with the other warps of the cluster (atomic max of the bits of a
// positive double).  Exact: a pruned chunk cannot hold a candidate scoring >=
// an existing one, so neither the argmax nor a tie is lost.  At most
// 32 * kMaxRounds chunks; every lane returns the same candidate.
constexpr int kMaxRounds = 3;
__device__ __forceinline__ Cand warp_range_best(const uint32_t *__restrict__ t, const uint64_t *__restrict__ PS1,
                                                const uint32_t *__restrict__ TB, uint64_t lo, uint64_t n, uint64_t S,
                                                uint64_t base, uint64_t r0, uint64_t r1,
                                                unsigned long long *cthr) {
    const int lane = threadIdx.x & 31;
    const double up = 1.0 + 0x1p-44, dn = 1.0 - 0x1p-44;
    const uint64_t q0 = r0 >> kChunkLog, nq = ((r1 - 1) >> kChunkLog) - q0 + 1;
    double d2[kMaxRounds], pm[kMaxRounds];
    uint64_t sla[kMaxRounds];
    double lbm = 0.0;
#pragma unroll
    for (int r = 0; r < kMaxRounds; r++) {   // loads of every round in flight first
        const uint64_t i = (uint64_t)r * 32 + lane;
        sla[r] = 0;
        pm[r] = 0.0;
        d2[r] = 0.0;
        if (i < nq) {
            const uint64_t q = q0 + i;
            sla[r] = PS1[q];
            const uint2 tb = reinterpret_cast<const uint2 *>(TB)[q];
            pm[r] = __longlong_as_double((long long)(((uint64_t)tb.y << 32) | tb.x));   // parked
        }
    }
#pragma unroll
    for (int r = 0; r < kMaxRounds; r++) {
        const uint64_t i = (uint64_t)r * 32 + lane;
        if (i < nq) {
            const uint64_t q = q0 + i;
            const uint64_t ra = max(r0, q << kChunkLog), rb = min(r1, (q + 1) << kChunkLog);
            const uint64_t pk = (uint64_t)__double_as_longlong(pm[r]);
            uint32_t ta = (uint32_t)(pk >> 32), tprev = (uint32_t)pk;
            uint64_t p = sla[r];
            if (ra & (kChunk - 1)) {   // unaligned start (the range's first chunk)
                for (uint64_t x = ra & ~(kChunk - 1); x < ra; x++) p += t[x];
                ta = t[ra];
                tprev = ra > lo ? t[ra - 1] : 0u;
            }
            const uint64_t SL = p - base;
            sla[r] = SL;
            const uint64_t ka = ra - lo, cnt = rb - ra;
            const u128 ad = (u128)S * ka - (u128)n * SL;
            const uint64_t nta = n * (uint64_t)ta;
            const double slope = S > nta ? __ull2double_rn(S - nta) : 0.0;
            const double dD = approx_d((uint32_t)(ad >> 64), (uint64_t)ad);
            const double dub = __dmul_rn(__dadd_rn(dD, __dmul_rn(slope, (double)(cnt - 1))), up);
            const uint64_t kf = max(ka, (uint64_t)1), kl = min(ka + cnt - 1, n - 1);
            pm[r] = 0.0;
            if (kf <= kl) {
                pm[r] = fmin(__dmul_rn((double)kf, (double)(n - kf)), __dmul_rn((double)kl, (double)(n - kl)));
                d2[r] = __dmul_rn(__dmul_rn(dub, dub), 1.0 + 0x1p-43);
            }
            if (ka >= 1 && tprev < ta)   // the chunk start is a real candidate
                lbm = fmax(lbm, div_lower(__dmul_rn(dD, dD), __dmul_rn((double)ka, (double)(n - ka))));
        }
    }
#pragma unroll
    for (int o = 16; o; o >>= 1) lbm = fmax(lbm, __shfl_xor_sync(0xffffffffu, lbm, o));
    double thr = __dmul_rn(lbm, dn);
    if (cthr) {
        unsigned long long prev = 0;
        if (lane == 0) prev = atomicMax(cthr, (unsigned long long)__double_as_longlong(thr));
        prev = __shfl_sync(0xffffffffu, prev, 0);
        thr = fmax(thr, __longlong_as_double((long long)prev));   // positive doubles order as integers
    }
    Cand best = no_cand();
    // kept when d2 >= thr * pmin (d2 = RN(dub^2) (1 + 2^-43) covers the roundings).
    // The round loop is rolled (per-round values picked by selects, not dynamic
    // register indexing) so the row scan appears once in the kernel body.
    // (Scanning the survivors four at a time with their rows loaded together
    // spilled registers and measured slower.)
#pragma unroll 1
    for (int r = 0; r < kMaxRounds; r++) {
        static_assert(kMaxRounds == 3, "the selects below cover three rounds");
        const double rd2 = r == 0 ? d2[0] : r == 1 ? d2[1] : d2[2];
        const double rpm = r == 0 ? pm[0] : r == 1 ? pm[1] : pm[2];
        const uint64_t rsl = r == 0 ? sla[0] : r == 1 ? sla[1] : sla[2];
        uint32_t live = __ballot_sync(0xffffffffu, rd2 > 0.0 && rd2 >= __dmul_rn(thr, rpm));
        while (live) {
            const int src = __ffs(live) - 1;
            live &= live - 1;
            const double sd2 = __shfl_sync(0xffffffffu, rd2, src), spm = __shfl_sync(0xffffffffu, rpm, src);
            if (sd2 < __dmul_rn(thr, spm)) continue;   // threshold raised meanwhile
            const uint64_t q = q0 + (uint64_t)r * 32 + src;
            const uint64_t SLa = __shfl_sync(0xffffffffu, rsl, src);
            scan_chunk(t, lo, n, S, max(r0, q << kChunkLog), min(r1, (q + 1) << kChunkLog), SLa, best);
            double lb = best.k ? div_lower(best.x, best.dp) : 0.0;
#pragma unroll
            for (int o = 16; o; o >>= 1) lb = fmax(lb, __shfl_xor_sync(0xffffffffu, lb, o));
            thr = fmax(thr, __dmul_rn(lb, dn));
        }
    }
#pragma unroll 1   // one copy of better() (with its 256-bit tie path) in the kernel body
    for (int o = 16; o; o >>= 1) {
        const Cand v = shfl_cand_xor(best, o);
        if (better(v, best)) best = v;
    }
    return best;
}

// warp: sum of t before lo (pref1(lo) = PS1[lo / 32] + partial chunk)
__device__ __forceinline__ uint64_t warp_pref1(const uint32_t *__restrict__ t, const uint64_t *__restrict__ PS1,
                                               uint64_t lo) {
    const int lane = threadIdx.x & 31;
    uint64_t part = 0;
    const uint64_t b0 = lo & ~(kChunk - 1);
    if (b0 + lane < lo) part = t[b0 + lane];
#pragma unroll
    for (int o = 16; o; o >>= 1) part += __shfl_xor_sync(0xffffffffu, part, o);
    return part + PS1[lo >> kChunkLog];
}

// Best valid cut of a whole cluster: the plain scan for <= 64 rows, chunk bounds
// up to 32 * kMaxRounds chunks, else the plain scan (only reached when
// big_rows() is raised past kSeg).
__device__ __forceinline__ Cand warp_best_cut(const uint32_t *__restrict__ t, const uint64_t *__restrict__ PS1,
                                              const uint32_t *__restrict__ TB, uint64_t lo, uint64_t n, uint64_t S) {
    const uint64_t nq = ((lo + n - 1) >> kChunkLog) - (lo >> kChunkLog) + 1;
    if (n <= 64 || nq > 32 * kMaxRounds) return warp_scan_cut(t, lo, n, S);
    return warp_range_best(t, PS1, TB, lo, n, S, warp_pref1(t, PS1, lo), lo, lo + n, nullptr);
}

// ---------------------------------------------------------------- mid clusters: a warp per cluster
// Clusters of local_rows() .. big_rows() rows, one warp each (grid-stride).
template <int MINB>
__global__ void __launch_bounds__(256, MINB) small_split_kernel(const uint32_t *__restrict__ f_lo,
                                                          const uint32_t *__restrict__ f_hi,
                                                          const uint64_t *__restrict__ f_S, const uint64_t *ctot,
                                                          const uint32_t *__restrict__ t,
                                                          const uint64_t *__restrict__ PS1,
                                                          const uint32_t *__restrict__ TB, uint32_t *__restrict__ cut,
                                                          uint64_t *__restrict__ cut_SL) {
    const uint32_t C = (uint32_t)(*ctot >> 32);   // frontier size, read on the device (pipelined levels)
    const int lane = threadIdx.x & 31;
    const uint64_t nwarps = ((uint64_t)gridDim.x * blockDim.x) >> 5;
    for (uint64_t c = ((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; c < C; c += nwarps) {
        const uint64_t lo = f_lo[c], n = f_hi[c] - lo;
        if (n < c_loc || n >= c_big) continue;
        const Cand best = warp_best_cut(t, PS1, TB, lo, n, f_S[c]);
        if (lane == 0) {
            cut[c] = best.k;
            cut_SL[c] = best.SL;
        }
    }
}

// ---------------------------------------------------------------- nearest-centre descent (exact, any size)
// The optimal cut k* of a cluster satisfies the nearest-centre condition of
// 2-means: t[k*-1] <= m(k*) <= t[k*], m(k) = (mu_L(k) + mu_R(k)) / 2.  (If
// t[k*-1] > m, the run of rows equal to t[k*-1] is strictly closer to mu_R:
// moving it to R is a valid cut with a strictly smaller within-cluster sum of
// squares, i.e. a strictly larger D^2 / (k (n - k)); symmetrically for t[k*].)
// Every maximiser, so every tie, satisfies it.  For sorted rows mu_L and mu_R,
// hence m, are non-decreasing in k, so a range of cuts [a, b] can hold a
// maximiser only if m(b) >= t[a-1] and m(a) <= t[b], and only if it holds a
// valid cut (t[a-1] < t[b]).  With cuts at 32-row chunk starts S_L is exact
// from the sampled prefix PS1 and t[a-1], t[b] come from the chunk-boundary
// pairs TB, so a warp tests 32 sub-ranges per step: a 32-ary descent from the
// whole cluster to the surviving 32-row chunks, which are scanned row by row
// (eval_cut, exact, ties -> smallest k).  All comparisons are exact integers:
// m(k) >= v  <=>  S_L (n - k) + (S - S_L) k >= 2 v k (n - k)  (both < 2^97).
__device__ __forceinline__ bool mid_ge(uint64_t SL, uint64_t k, uint64_t n, uint64_t S, uint32_t v) {
    const uint64_t nk = n - k;
    const u128 F = (u128)SL * nk + (u128)(S - SL) * k;
    const u128 G = (u128)(k * nk) * (2ull * v);
    return F >= G;
}
__device__ __forceinline__ bool mid_le(uint64_t SL, uint64_t k, uint64_t n, uint64_t S, uint32_t v) {
    const uint64_t nk = n - k;
    const u128 F = (u128)SL * nk + (u128)(S - SL) * k;
    const u128 G = (u128)(k * nk) * (2ull * v);
    return F <= G;
}

#ifndef SR_NC_MINB
#define SR_NC_MINB 9
#endif
#ifndef SR_NC_THREADS
#define SR_NC_THREADS 128
#endif
#ifndef SR_NC_SBEST
#define SR_NC_SBEST 1
#endif
#ifndef SR_NC_QUEUE
#define SR_NC_QUEUE 1
#endif
constexpr int kNcStack = 256;   // per warp: 1 + 31 x (descent depth <= 6) entries suffice
struct NcStats {
    unsigned long long *n_nodes, *n_scanned;
};
__global__ void __launch_bounds__(SR_NC_THREADS, SR_NC_MINB) nc_split_kernel(const uint32_t *__restrict__ f_lo,
                                                       const uint32_t *__restrict__ f_hi,
                                                       const uint64_t *__restrict__ f_S, const uint64_t *ctot,
                                                       const uint32_t *__restrict__ t,
                                                       const uint64_t *__restrict__ PS1,
                                                       const uint32_t *__restrict__ TB, uint32_t *__restrict__ cut,
                                                       uint64_t *__restrict__ cut_SL, uint64_t nmin, NcStats st,
                                                       uint32_t *__restrict__ queue, uint32_t *__restrict__ queue_next,
                                                       uint64_t *__restrict__ ntot) {
    __shared__ uint2 s_stack[SR_NC_THREADS / 32][kNcStack];
#if SR_NC_SBEST
    __shared__ Cand s_best[SR_NC_THREADS / 32][32];   // each lane's best candidate lives in shared memory (registers for occupancy)
#endif
    const uint32_t C = (uint32_t)(*ctot >> 32);
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    if (blockIdx.x == 0 && threadIdx.x == 0) {   // for the next kernels in stream order (no memset launches)
        if (queue_next) *queue_next = 0u;    // the next level's work queue
        if (ntot) *ntot = 0ull;              // the frontier this level's decision appends to
    }
    uint2 *stk = s_stack[w];
    const uint2 *TB2 = reinterpret_cast<const uint2 *>(TB);
    const uint32_t nwarps = (gridDim.x * blockDim.x) >> 5;
    uint32_t my_nodes = 0, my_scanned = 0;
    // clusters by a work queue (the next index fetched while this one is split:
    // cluster sizes vary by orders of magnitude) or grid-stride
    uint32_t c = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    for (; c < C;) {
        uint32_t cn = 0;
        if (SR_NC_QUEUE && lane == 0) cn = nwarps + atomicAdd(queue, 1u);
        const uint32_t lo = f_lo[c], hi = f_hi[c], n = hi - lo;
        if (n < nmin) {
            c = SR_NC_QUEUE ? __shfl_sync(0xffffffffu, cn, 0) : c + nwarps;
            continue;
        }
        const uint64_t S = f_S[c];
        const uint64_t base = warp_pref1(t, PS1, lo);
#if SR_NC_SBEST
        Cand &best = s_best[w][lane];
#else
        Cand best;
#endif
        best = no_cand();
        // aligned chunks [C0, C1]: cut positions 32 C0 .. 32 C1 + 31 within [lo + 1, hi - 2],
        // and the next chunk start 32 (C1 + 1) <= hi - 1 (so m is defined there)
        const uint32_t C0 = (uint32_t)(((uint64_t)lo + kChunk) >> kChunkLog);
        const int64_t C1s = ((int64_t)hi - 33) >> kChunkLog;
        if (hi < 33 || (int64_t)C0 > C1s) {   // short: scan every cut
            uint64_t SLa = 0;
            for (uint64_t ra = lo; ra < hi; ra += 32) {
                const uint64_t rb = min(ra + 32, (uint64_t)hi);
                scan_chunk(t, lo, n, S, ra, rb, SLa, best);
                uint64_t v = ra + lane < rb ? t[ra + lane] : 0u;
#pragma unroll
                for (int o = 16; o; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
                SLa += v;
            }
            my_scanned += (uint32_t)((n + 31) / 32);
        } else {
            const uint32_t C1 = (uint32_t)C1s;
            // head cuts [lo + 1, 32 C0) and tail cuts [32 (C1 + 1), hi)
            scan_chunk(t, lo, n, S, lo, (uint64_t)C0 << kChunkLog, 0, best);
            scan_chunk(t, lo, n, S, (uint64_t)(C1 + 1) << kChunkLog, hi, PS1[C1 + 1] - base, best);
            int sp = 0;
            if (lane == 0) stk[0] = make_uint2(C0, C1);
            sp = 1;
            __syncwarp();
            while (sp > 0) {
                const uint2 nd = stk[--sp];
                __syncwarp();
                const uint32_t c0 = nd.x, c1 = nd.y;
                const uint32_t wd = (c1 - c0 + 32) / 32;          // chunks per sub-range
                const uint32_t s0 = c0 + (uint32_t)lane * wd;
                const bool in = s0 <= c1;
                const uint32_t s1 = min(s0 + wd - 1, c1);
                bool keep = false;
                uint64_t SLs = 0;
                if (in) {
                    SR_DCHECK(s0 >= C0 && s1 + 1 <= (uint32_t)C1s + 1 && ((uint64_t)(s1 + 1) << kChunkLog) < hi);
                    const uint64_t pa = PS1[s0], pb = PS1[s1 + 1];
                    const uint32_t tam1 = TB2[s0].x, tb = TB2[s1 + 1].x;   // t[32 s0 - 1], t[32 s1 + 31]
                    SLs = pa - base;
                    const uint64_t ka = ((uint64_t)s0 << kChunkLog) - lo, kb = ((uint64_t)(s1 + 1) << kChunkLog) - lo;
                    keep = tam1 < tb && mid_ge(pb - base, kb, n, S, tam1) && mid_le(SLs, ka, n, S, tb);
                }
                my_nodes += in ? 1u : 0u;
                uint32_t live = __ballot_sync(0xffffffffu, keep);
                if (wd == 1) {   // single chunks: scan the survivors now
                    while (live) {
                        const int src = __ffs(live) - 1;
                        live &= live - 1;
                        const uint64_t q = c0 + (uint64_t)src;
                        const uint64_t SLa = __shfl_sync(0xffffffffu, SLs, src);
                        scan_chunk(t, lo, n, S, q << kChunkLog, (q + 1) << kChunkLog, SLa, best);
                        my_scanned++;
                    }
                } else {
                    const int below = __popc(live & ((1u << lane) - 1));
                    SR_DCHECK(sp + __popc(live) <= kNcStack);
                    if (keep) stk[sp + __popc(live) - 1 - below] = make_uint2(s0, s1);   // leftmost on top
                    sp += __popc(live);
                    __syncwarp();
                }
            }
        }
        Cand fin = best;
#pragma unroll 1   // one copy of better() (with its 256-bit tie path) in the kernel body
        for (int o = 16; o; o >>= 1) {
            const Cand v = shfl_cand_xor(fin, o);
            if (better(v, fin)) fin = v;
        }
        if (lane == 0) {
            cut[c] = fin.k;
            cut_SL[c] = fin.SL;
        }
        c = SR_NC_QUEUE ? __shfl_sync(0xffffffffu, cn, 0) : c + nwarps;
    }
    // stats (lane sums; scanned is warp-uniform)
    for (int o = 16; o; o >>= 1) my_nodes += __shfl_xor_sync(0xffffffffu, my_nodes, o);
    if (lane == 0 && my_nodes) {
        atomicAdd(st.n_nodes, (unsigned long long)my_nodes);
        atomicAdd(st.n_scanned, (unsigned long long)my_scanned);
    }
}

// ---------------------------------------------------------------- split variant: Lloyd (R26)
// Lloyd's k-means with k = 2 ("k-means", P:L258 k = 2) from the (min, max)
// centroids to its fixed point, one warp per cluster.  On sorted rows an
// assignment is a cut: cluster 1 = the rows with 2 t <= c1 + c2, i.e. with the
// exact fractional centroids c1 = S1/k, c2 = S2/(n-k), t * 2k(n-k) <= S1 (n-k)
// + S2 k (integers < 2^97).  The cut is found by a 33-ary search (32 probes per
// warp round trip), S1 from the sampled prefix; at most kLloydMaxIters
// assignment steps (the bound DESIGN.md R26 states for both sides).
constexpr uint32_t kLloydMaxIters = 1000;

// first row in [a, b) whose t fails t * f <= rhs (rows sorted by t, so the
// rows passing the test form a prefix); every lane returns it
__device__ __forceinline__ uint64_t warp_cut_search(const uint32_t *__restrict__ t, uint64_t a, uint64_t b, uint64_t f,
                                                    u128 rhs) {
    const int lane = threadIdx.x & 31;
    while (b - a > 32) {
        const uint64_t p = a + ((uint64_t)(lane + 1) * (b - a)) / 33;
        const uint32_t m = __ballot_sync(0xffffffffu, (u128)t[p] * f <= rhs);
        const int c = __popc(m);   // a prefix of the probes passes
        const uint64_t pa = __shfl_sync(0xffffffffu, p, c > 0 ? c - 1 : 0), pb = __shfl_sync(0xffffffffu, p, c < 32 ? c : 31);
        if (c > 0) a = pa + 1;
        if (c < 32) b = pb;
    }
    const uint32_t m = __ballot_sync(0xffffffffu, a + lane < b && (u128)t[a + lane] * f <= rhs);
    return a + __popc(m);
}

// k-means++ seeds (split = 2, reading R27): the D^2 draw of the second seed is
// the first row r of the cluster whose running sum W(r + 1 - lo), W(p) =
// sum_{i < p} (t_i - c1)^2 = Q(p) + p c1^2 - 2 c1 S(p), exceeds R.  W is
// monotone, so a warp 33-ary search over the 32-row chunk boundaries inside the
// cluster (exact W from PS1/PS2 alone, two loads per probe) finds the chunk
// holding r, and one warp scan of that chunk's (t - c1)^2 finds r.  Returns r
// relative to lo.
__device__ __forceinline__ uint64_t warp_d2_search(const uint32_t *__restrict__ t, const uint64_t *__restrict__ PS1,
                                                   const u128 *__restrict__ PS2, uint64_t lo, uint64_t hi,
                                                   uint64_t s0, u128 q0, uint32_t c1, u128 R) {
    const int lane = threadIdx.x & 31;
    const u128 cc = (u128)((uint64_t)c1 * c1);
    const u128 c2x = (u128)(2 * (uint64_t)c1);
    auto W_at = [&](uint64_t j) {   // W at the chunk boundary 32 j (lo < 32 j <= hi)
        return (PS2[j] - q0) + cc * ((j << kChunkLog) - lo) - c2x * (PS1[j] - s0);
    };
    // boundaries 32 j with lo < 32 j <= hi: j in [jlo, jhi]; first j with W > R
    const uint64_t jlo = (lo >> kChunkLog) + 1, jhi = hi >> kChunkLog;
    uint64_t a = jlo, b = jhi + 1;
    while (b - a > 32) {
        const uint64_t p = a + ((uint64_t)(lane + 1) * (b - a)) / 33;
        const uint32_t m = __ballot_sync(0xffffffffu, W_at(p) <= R);
        const int c = __popc(m);
        const uint64_t pa = __shfl_sync(0xffffffffu, p, c > 0 ? c - 1 : 0), pb = __shfl_sync(0xffffffffu, p, c < 32 ? c : 31);
        if (c > 0) a = pa + 1;
        if (c < 32) b = pb;
    }
    const uint32_t m = __ballot_sync(0xffffffffu, a + lane < b && W_at(a + lane) <= R);
    const uint64_t jf = a + __popc(m);
    // r lies in the rows [ra, rb) between the last boundary at or below R and the first above it
    const uint64_t ra = jf > jlo ? (jf - 1) << kChunkLog : lo, rb = jf <= jhi ? jf << kChunkLog : hi;
    const u128 Wa = jf > jlo ? W_at(jf - 1) : (u128)0;
    const uint64_t row = ra + lane;
    const bool in = row < rb;
    uint64_t d = 0;
    if (in) {
        const uint32_t x = t[row];
        d = x > c1 ? (uint64_t)(x - c1) : (uint64_t)(c1 - x);
    }
    // inclusive warp scan of d^2 (< 2^64 each) in 128 bits
    uint64_t slo = d * d, shi = 0;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const uint64_t vlo = __shfl_up_sync(0xffffffffu, slo, o), vhi = __shfl_up_sync(0xffffffffu, shi, o);
        if (lane >= o) {
            const uint64_t nlo = slo + vlo;
            shi += vhi + (nlo < slo ? 1 : 0);
            slo = nlo;
        }
    }
    const u128 run = Wa + (((u128)shi << 64) | slo);
    const uint32_t over = __ballot_sync(0xffffffffu, in && run > R);
    return ra + (uint64_t)(__ffs(over) - 1) - lo;
}

template <bool PP>
__global__ void __launch_bounds__(256) lloyd_split_kernel(const uint32_t *__restrict__ f_lo, const uint32_t *__restrict__ f_hi,
                                                          const uint64_t *__restrict__ f_S, const u128 *__restrict__ f_Q,
                                                          const uint64_t *ctot, const uint32_t *__restrict__ t,
                                                          const uint64_t *__restrict__ PS1, const u128 *__restrict__ PS2,
                                                          uint32_t k0, uint32_t k1, uint32_t *__restrict__ cut,
                                                          uint64_t *__restrict__ cut_SL, uint32_t *__restrict__ queue) {
    const uint32_t C = (uint32_t)(*ctot >> 32);
    const int lane = threadIdx.x & 31;
    const uint32_t nwarps = (gridDim.x * blockDim.x) >> 5;
    // clusters from a work queue (the next index fetched while this one is split)
    for (uint32_t c = (blockIdx.x * blockDim.x + threadIdx.x) >> 5, cn = 0; c < C; c = __shfl_sync(0xffffffffu, cn, 0)) {
        if (lane == 0) cn = nwarps + atomicAdd(queue, 1u);
        const uint64_t lo = f_lo[c], hi = f_hi[c], n = hi - lo, S = f_S[c];
        uint64_t base;
        u128 mid2;
        if (PP) {   // R27: c1 a uniform row, c2 by D^2 weight (one Philox draw per cluster)
            const U4 x = philox4x32_10(U4{t[lo], t[hi - 1], (uint32_t)n, 0x4B4D5050u}, k0, k1);
            const uint64_t j1 = (uint64_t)(((u128)(((uint64_t)x.y << 32) | x.x) * n) >> 64);
            const uint32_t c1 = t[lo + j1];
            const u128 W = (f_Q[c] + (u128)((uint64_t)c1 * c1) * n) - (u128)(2 * (uint64_t)c1) * S;
            const u128 R = (W * x.z) >> 32;
            u128 q0;
            pref12(PS1, PS2, t, lo, base, q0);
            const uint64_t j2 = warp_d2_search(t, PS1, PS2, lo, hi, base, q0, c1, R);
            mid2 = (u128)c1 + t[lo + j2];
        } else {    // R26: centroids (min, max)
            base = pref1(PS1, t, lo);
            mid2 = (u128)t[lo] + t[hi - 1];
        }
        // first assignment 2 t <= c1 + c2
        uint64_t k = warp_cut_search(t, lo, hi, 2, mid2) - lo;
        uint64_t S1 = 0;
        for (uint32_t it = 1;; it++) {
            S1 = pref1(PS1, t, lo + k) - base;   // step 3: exact centroid sums
            if (it >= kLloydMaxIters) break;
            const u128 rhs = (u128)S1 * (n - k) + (u128)(S - S1) * k;
            const uint64_t k2 = warp_cut_search(t, lo, hi, 2 * k * (n - k), rhs) - lo;
            if (k2 == k) break;
            k = k2;
        }
        if (lane == 0) {
            cut[c] = (uint32_t)k;
            cut_SL[c] = S1;
        }
    }
}

// ---------------------------------------------------------------- big clusters: chunk bounds
// Clusters of >= kBig rows.  One block per kBigSeg rows.  For every 32-row chunk
// (aligned to the sampled prefix PS1) the concavity bound of |D| gives an upper
// bound of the chunk's scores from S_L at the chunk start (PS1, exact) and one
// t value; a real candidate at every chunk start gives lower bounds.  Only
// chunks whose bound reaches the best lower bound (of this block, or of the
// whole cluster through an atomic max) are scanned row by row.  Exact: a pruned
// chunk cannot hold a candidate scoring >= an existing one, so neither the
// argmax nor a tie is lost.
struct BigEntry {
    uint32_t c, seg;
};

__device__ __forceinline__ uint32_t big_nseg(uint64_t lo, uint64_t hi) {
    return (uint32_t)((hi - lo + kBigSeg - 1) / kBigSeg);
}

__global__ void big_entries_kernel(const uint32_t *__restrict__ f_lo, const uint32_t *__restrict__ f_hi,
                                   const uint64_t *ctot, BigEntry *__restrict__ ent, uint32_t *__restrict__ first_ent,
                                   uint32_t *__restrict__ count, unsigned long long *__restrict__ thr) {
    const uint64_t c = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (c >= (*ctot >> 32)) return;
    thr[c] = 0;   // the cluster's pruning threshold (seeded and raised by the big-path kernels)
    const uint64_t n = f_hi[c] - f_lo[c];
    if (n < c_big) return;
    const uint32_t nb = big_nseg(f_lo[c], f_hi[c]);
    const uint32_t e0 = atomicAdd(count, nb);
    for (uint32_t s = 0; s < nb; s++) ent[e0 + s] = BigEntry{(uint32_t)c, s};
    first_ent[c] = e0;
}

struct BigArgs {
    const BigEntry *ent;
    const uint32_t *count;
    const uint32_t *f_lo, *f_hi;
    const uint64_t *f_S, *PS1;
    const uint32_t *t;
    const uint32_t *TB;        // chunk-boundary pairs (t[32 j - 1], t[32 j])
    unsigned long long *thr;   // per cluster: bits of the best lower bound so far
    Cand *part;                // per entry
    unsigned long long *n_chunks, *n_scanned;   // stats
};

constexpr int kBigThreads = 256;

// Seed of each big cluster's pruning threshold: real candidates on a coarse
// grid (every kSeedStride rows, at chunk starts, so S_L comes from PS1 and the
// validity t[k-1] < t[k] from TB), one warp per entry.  Their best lower bound
// (atomic max of the bits of a positive double) is a strict lower bound of a
// real candidate's score, so pruning against it keeps the argmax and its ties;
// it only makes far-away segments prune as hard as the segment holding the
// optimum.
constexpr uint64_t kSeedStride = 1024;
__global__ void __launch_bounds__(256) big_seed_kernel(BigArgs a) {
    const uint32_t n_ent = *a.count;
    const int lane = threadIdx.x & 31;
    const uint32_t nw = gridDim.x * (blockDim.x / 32);
    for (uint32_t eb = blockIdx.x * (blockDim.x / 32) + (threadIdx.x >> 5); eb < n_ent; eb += nw) {
        const BigEntry e = a.ent[eb];
        const uint64_t lo = a.f_lo[e.c], hi = a.f_hi[e.c], n = hi - lo, S = a.f_S[e.c];
        const uint64_t r0 = lo + (uint64_t)e.seg * kBigSeg, r1 = min(r0 + kBigSeg, hi);
        uint64_t part = 0;
        const uint64_t lb0 = lo & ~(kChunk - 1);
        if (lb0 + lane < lo) part = a.t[lb0 + lane];
#pragma unroll
        for (int o = 16; o; o >>= 1) part += __shfl_xor_sync(0xffffffffu, part, o);
        const uint64_t base = a.PS1[lo >> kChunkLog] + part;
        const uint64_t g0 = (r0 + kChunk - 1) & ~(kChunk - 1);   // first chunk start in the segment
        double lbm = 0.0;
#pragma unroll
        for (int r = 0; r < (int)(kBigSeg / kSeedStride / 32); r++) {
            const uint64_t ra = g0 + ((uint64_t)r * 32 + lane) * kSeedStride;
            if (ra > lo && ra < r1) {
                const uint64_t SL = a.PS1[ra >> kChunkLog] - base;
                const uint2 tb = reinterpret_cast<const uint2 *>(a.TB)[ra >> kChunkLog];
                if (tb.x < tb.y) {   // t[ra - 1] < t[ra]: a valid cut
                    const uint64_t ka = ra - lo;
                    const u128 ad = (u128)S * ka - (u128)n * SL;
                    const double dD = approx_d((uint32_t)(ad >> 64), (uint64_t)ad);
                    lbm = fmax(lbm, div_lower(__dmul_rn(dD, dD), __dmul_rn((double)ka, (double)(n - ka))));
                }
            }
        }
#pragma unroll
        for (int o = 16; o; o >>= 1) lbm = fmax(lbm, __shfl_xor_sync(0xffffffffu, lbm, o));
        if (lane == 0 && lbm > 0.0)
            atomicMax(a.thr + e.c, (unsigned long long)__double_as_longlong(__dmul_rn(lbm, 1.0 - 0x1p-44)));
    }
}
constexpr int kBigChunks = (int)(kBigSeg / kChunk) + 2;
constexpr int kBigRounds = (kBigChunks + kBigThreads - 1) / kBigThreads;
constexpr size_t kBigSmem = (size_t)kBigChunks * (sizeof(double) + sizeof(uint64_t) + sizeof(uint2) + sizeof(float) +
                                                  sizeof(uint16_t));

#ifndef SR_BIG_MINB
#define SR_BIG_MINB 3
#endif
__global__ void __launch_bounds__(kBigThreads, SR_BIG_MINB) big_split_kernel(BigArgs a) {
    extern __shared__ __align__(16) unsigned char s_big[];   // kBigSmem bytes
    double *s_ub = reinterpret_cast<double *>(s_big);          // d2: the squared |D| bound of the chunk
    uint64_t *s_sl = reinterpret_cast<uint64_t *>(s_ub + kBigChunks);   // PS1 at the chunk start, then S_L
    uint2 *s_tb = reinterpret_cast<uint2 *>(s_sl + kBigChunks);         // TB pair at the chunk start
    float *s_pm = reinterpret_cast<float *>(s_tb + kBigChunks);         // min k (n - k), rounded down (prunes less)
    uint16_t *s_list = reinterpret_cast<uint16_t *>(s_pm + kBigChunks);
    __shared__ uint32_t s_nlist;
    __shared__ double s_thr[kBigThreads / 32];
    __shared__ Cand s_best[kBigThreads / 32];
    __shared__ uint64_t s_base;
    const uint32_t n_ent = *a.count;
    const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
    // the entry descriptors are software-pipelined: the next entry's (cluster,
    // lo, hi, S) loads are issued while the current entry is processed
    BigEntry e{0, 0};
    uint64_t lo = 0, hi = 0, S = 0;
    if (blockIdx.x < n_ent) {
        e = a.ent[blockIdx.x];
        lo = a.f_lo[e.c];
        hi = a.f_hi[e.c];
        S = a.f_S[e.c];
    }
    for (uint32_t eb = blockIdx.x; eb < n_ent; eb += gridDim.x) {
    __syncthreads();   // shared memory of the previous entry
    const uint64_t n = hi - lo;
    const uint64_t r0 = lo + (uint64_t)e.seg * kBigSeg, r1 = min(r0 + kBigSeg, hi);
    const uint64_t q0 = r0 >> kChunkLog, q1 = (r1 - 1) >> kChunkLog;   // chunks touching [r0, r1)
    const int nq = (int)(q1 - q0 + 1);
    const double up = 1.0 + 0x1p-44, dn = 1.0 - 0x1p-44;
    double lbm = 0.0;
    // every round's sampled-prefix and boundary loads in flight first (staged
    // in shared memory, so the bound loop below stays rolled: a small kernel
    // body, the unrolled one missed the instruction cache), with pref1(lo) and
    // the next entry's descriptors
#pragma unroll
    for (int r = 0; r < kBigRounds; r++) {
        const int i = tid + r * kBigThreads;
        if (i < nq) {
            s_sl[i] = a.PS1[q0 + i];
            s_tb[i] = reinterpret_cast<const uint2 *>(a.TB)[q0 + i];
        }
    }
    if (w == 0) {   // pref1(lo) = PS1[lo/32] + partial chunk
        uint64_t part = 0;
        const uint64_t lb0 = lo & ~(kChunk - 1);
        if (lb0 + lane < lo) part = a.t[lb0 + lane];
        const uint64_t p1 = a.PS1[lo >> kChunkLog];
        for (int o = 16; o; o >>= 1) part += __shfl_xor_sync(0xffffffffu, part, o);
        if (lane == 0) {
            s_base = p1 + part;
            s_nlist = 0;
        }
    }
    const uint32_t ebn = eb + gridDim.x;
    BigEntry en{0, 0};
    uint64_t lon = 0, hin = 0, Sn = 0;
    if (ebn < n_ent) {
        en = a.ent[ebn];
        lon = a.f_lo[en.c];
        hin = a.f_hi[en.c];
        Sn = a.f_S[en.c];
    }
    __syncthreads();
#pragma unroll 1
    for (int i = tid; i < nq; i += kBigThreads) {
        const uint64_t q = q0 + i;
        const uint64_t ra = max(r0, q << kChunkLog), rb = min(r1, (q + 1) << kChunkLog);   // rows [ra, rb)
        uint64_t pa = s_sl[i];
        const bool al = (ra & (kChunk - 1)) == 0;
        if (!al)   // only the block's first chunk can start unaligned
            for (uint64_t x = ra & ~(kChunk - 1); x < ra; x++) pa += a.t[x];
        const uint64_t SL = pa - s_base;       // S_L at k_a = ra - lo (exact)
        const uint32_t ka = (uint32_t)(ra - lo);
        const uint2 tb = al ? s_tb[i] : make_uint2(0u, 0u);
        const uint32_t ta = al ? tb.y : a.t[ra];
        s_sl[i] = SL;
        const u128 ad = (u128)S * ka - (u128)n * SL;
        const uint64_t cnt = rb - ra;
        bool has_e = false;
        double E = 0.0;
        uint32_t tl = 0;
        if (c_bound2) {
            if (rb == hi) {                          // ad = 0 at the cluster end
                has_e = true;
                tl = a.t[rb - 1];
            } else if ((rb & (kChunk - 1)) == 0) {   // the next chunk's start (sampled prefix)
                has_e = true;
                const u128 ade = (u128)S * (rb - lo) - (u128)n * (a.PS1[rb >> kChunkLog] - s_base);
                E = approx_d((uint32_t)(ade >> 64), (uint64_t)ade);
                tl = reinterpret_cast<const uint2 *>(a.TB)[rb >> kChunkLog].x;
            }
        }
        const double dub =
            __dmul_rn(chunk_ad_bound(approx_d((uint32_t)(ad >> 64), (uint64_t)ad), n, S, ta, cnt, has_e, E, tl), up);
        const uint64_t kf = max((uint64_t)ka, (uint64_t)1), kl = min((uint64_t)ka + cnt - 1, n - 1);
        // division-free: the chunk survives when d2 >= thr * pmin, d2 = RN(dub^2) (1 + 2^-43)
        // covering the roundings (as warp_range_best)
        double d2 = 0.0, pmin = 0.0;
        if (kf <= kl) {
            pmin = fmin(__dmul_rn((double)kf, (double)(n - kf)), __dmul_rn((double)kl, (double)(n - kl)));
            d2 = __dmul_rn(__dmul_rn(dub, dub), 1.0 + 0x1p-43);
        }
        s_ub[i] = d2;
        s_pm[i] = __double2float_rd(pmin);
        if (ka >= 1 && (al ? tb.x : a.t[ra - 1]) < ta) {   // the chunk start is a real candidate
            const double dD = approx_d((uint32_t)(ad >> 64), (uint64_t)ad);
            lbm = fmax(lbm, div_lower(__dmul_rn(dD, dD), __dmul_rn((double)ka, (double)(n - ka))));
        }
    }
    for (int o = 16; o; o >>= 1) lbm = fmax(lbm, __shfl_xor_sync(0xffffffffu, lbm, o));
    if (lane == 0) s_thr[w] = lbm;
    __syncthreads();
    if (tid == 0) {   // block best vs the cluster's threshold (positive doubles order as integers)
        double m = 0.0;
        for (int k = 0; k < kBigThreads / 32; k++) m = fmax(m, s_thr[k]);
        const unsigned long long prev = atomicMax(a.thr + e.c, (unsigned long long)__double_as_longlong(m));
        s_thr[0] = fmax(m, __longlong_as_double((long long)prev));
    }
    __syncthreads();
    const double thr = __dmul_rn(s_thr[0], dn);
    for (int i = tid; i < nq; i += kBigThreads)
        if (s_ub[i] > 0.0 && s_ub[i] >= __dmul_rn(thr, (double)s_pm[i])) s_list[atomicAdd(&s_nlist, 1u)] = (uint16_t)i;
    __syncthreads();
    if (tid == 0) {   // stats: chunks bounded / scanned
        atomicAdd(a.n_chunks, (unsigned long long)nq);
        atomicAdd(a.n_scanned, (unsigned long long)s_nlist);
    }
    // row-by-row scan of the surviving chunks: one warp per chunk, lane = row;
    // kScanU chunks per warp step with their loads in flight first
    constexpr int kScanU = 4, kNW = kBigThreads / 32;
    Cand best = no_cand();
    const uint32_t nlist = s_nlist;
    for (uint32_t lb = w; lb < nlist; lb += kNW * kScanU) {
        uint32_t tcv[kScanU], tpv[kScanU];
#pragma unroll
        for (int u = 0; u < kScanU; u++) {
            const uint32_t li = lb + u * kNW;
            tcv[u] = 0u;
            tpv[u] = 0u;
            if (li < nlist) {
                const uint64_t q = q0 + s_list[li];
                const uint64_t ra = max(r0, q << kChunkLog), rb = min(r1, (q + 1) << kChunkLog);
                const uint64_t row = ra + lane;
                if (row < rb) tcv[u] = a.t[row];
                if (lane == 0 && row > lo) tpv[u] = a.t[row - 1];
            }
        }
#pragma unroll
        for (int u = 0; u < kScanU; u++) {
            const uint32_t li = lb + u * kNW;
            if (li >= nlist) break;
            const int i = s_list[li];
            const uint64_t q = q0 + i;
            const uint64_t ra = max(r0, q << kChunkLog), rb = min(r1, (q + 1) << kChunkLog);
            const uint64_t row = ra + lane;
            const bool in = row < rb;
            const uint32_t tc = tcv[u];
            uint32_t tp = __shfl_up_sync(0xffffffffu, tc, 1);
            if (lane == 0) tp = tpv[u];
            uint64_t incl = tc;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const uint64_t v = __shfl_up_sync(0xffffffffu, incl, o);
                if (lane >= o) incl += v;
            }
            const uint64_t SLr = s_sl[i] + incl - tc;
            const uint32_t k = (uint32_t)(row - lo);
            if (in && k >= 1 && tp < tc) eval_cut(k, n, S, SLr, best);
        }
    }
#pragma unroll 1   // one copy of better() (with its 256-bit tie path) in the kernel body
    for (int o = 16; o; o >>= 1) {
        const Cand v = shfl_cand_xor(best, o);
        if (better(v, best)) best = v;
    }
    if (lane == 0) s_best[w] = best;
    __syncthreads();
    if (tid == 0) {
        for (int k = 1; k < kBigThreads / 32; k++)
            if (better(s_best[k], best)) best = s_best[k];
        a.part[eb] = best;
    }
    e = en;
    lo = lon;
    hi = hin;
    S = Sn;
    }
}

// one block per big cluster: argmax over its entries
__global__ void big_reduce_kernel(const uint32_t *__restrict__ f_lo, const uint32_t *__restrict__ f_hi,
                                  const uint64_t *ctot, const uint32_t *__restrict__ first_ent,
                                  const Cand *__restrict__ part, uint32_t *__restrict__ cut,
                                  uint64_t *__restrict__ cut_SL) {
  const uint64_t C = *ctot >> 32;
  for (uint64_t c = blockIdx.x; c < C; c += gridDim.x) {
    const uint64_t n = f_hi[c] - f_lo[c];
    if (n < c_big) continue;
    const uint32_t nb = big_nseg(f_lo[c], f_hi[c]), e0 = first_ent[c];
    Cand best = no_cand();
    for (uint32_t s = threadIdx.x; s < nb; s += 32)
        if (better(part[e0 + s], best)) best = part[e0 + s];
#pragma unroll 1   // one copy of better() (with its 256-bit tie path) in the kernel body
    for (int o = 16; o; o >>= 1) {
        const Cand v = shfl_cand_xor(best, o);
        if (better(v, best)) best = v;
    }
    if (threadIdx.x == 0) {
        cut[c] = best.k;
        cut_SL[c] = best.SL;
    }
  }
}

// ---------------------------------------------------------------- a4: decide
struct DecideArgs {
    const uint32_t *f_lo, *f_hi, *cut;
    const uint64_t *f_S, *cut_SL;
    const u128 *f_Q;
    const uint64_t *ctot;   // packed (count << 32 | rows) of the current frontier
    const uint64_t *PS1;
    const u128 *PS2;
    const uint32_t *t;
    uint32_t *flags;   // leaf-start bitmap
    uint32_t *nlo, *nhi;   // next frontier
    uint64_t *nS;
    u128 *nQ;
    uint64_t *total;       // packed (count << 32 | rows) of the next frontier (zeroed before)
    double eps, z, k2;
    int clamp;
};

__device__ __forceinline__ double eq3_m(u128 V, uint64_t S, double k2, int clamp) {
    if (V == 0) return clamp ? 1.0 : 0.0;
    const double dS = rn64(S);
    double m = ceil(__dmul_rn(__ddiv_rn(rn128(V), __dmul_rn(dS, dS)), k2));
    if (clamp && m < 1.0) m = 1.0;
    return m;
}

__device__ __forceinline__ double eq6_m(double g, double mu, double V, int clamp) {
    if (V == 0.0) return clamp ? 1.0 : 0.0;
    double m = ceil(__dmul_rn(g, __dsqrt_rn(__ddiv_rn(V, mu))));
    if (clamp && m < 1.0) m = 1.0;
    return m;
}

// Eq. 7 vs Eq. 8 for a cluster (n, S, Q) cut at k (k >= 1) with left sums
// (SL, QL): true when the split lowers the sample cost (strict).
__device__ __forceinline__ bool split_pays(uint64_t n, uint64_t S, u128 Q, uint64_t k, uint64_t SL, u128 QL,
                                           double eps, double z, double k2, int clamp) {
    const uint64_t nL = k, nR = n - k, SR = S - SL;
    const u128 QR = Q - QL;
    const u128 V = (u128)n * Q - (u128)S * S;
    const u128 VL = (u128)nL * QL - (u128)SL * SL, VR = (u128)nR * QR - (u128)SR * SR;
    // Eq. 7: tau_old = m * Xbar, m from Eq. 3
    const double mu = __ddiv_rn(rn64(S), rn64(n));
    const double tau_old = __dmul_rn(eq3_m(V, S, k2, clamp), mu);
    // Eq. 8 with Eq. 6 (corrected numerator) over {L, R}, c from the parent's total
    const double muL = __ddiv_rn(rn64(SL), rn64(nL)), muR = __ddiv_rn(rn64(SR), rn64(nR));
    const double dVL = rn128(VL), dVR = rn128(VR);
    const double w = __ddiv_rn(__dmul_rn(eps, rn64(S)), z);
    const double cc = __dmul_rn(w, w);
    const double ssum = __dadd_rn(__dsqrt_rn(__dmul_rn(muL, dVL)), __dsqrt_rn(__dmul_rn(muR, dVR)));
    const double g = __ddiv_rn(ssum, cc);
    const double mL = eq6_m(g, muL, dVL, clamp), mR = eq6_m(g, muR, dVR, clamp);
    const double tau_new = __dadd_rn(__dmul_rn(mL, muL), __dmul_rn(mR, muR));
    return tau_new < tau_old;
}

// clusters of >= local_rows() rows (the local kernel finishes the others).
// Accepted cuts set their leaf-start bit, and the non-trivial children are
// appended to the next frontier directly: a warp-aggregated atomicAdd on the
// packed (count << 32 | rows) total gives each warp its slots.  The frontier
// order is immaterial (leaves come from the bitmap, decisions from each
// cluster's own rows), so no ordered compaction is needed.
__global__ void __launch_bounds__(256) decide_kernel(DecideArgs a) {
    const uint64_t c = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const int lane = threadIdx.x & 31;
    uint32_t lo = 0, hi = 0, mid = 0;
    uint64_t S = 0, SL = 0;
    u128 Q = 0, QL = 0;
    bool ntL = false, ntR = false;
    if (c < (*a.ctot >> 32)) {
        lo = a.f_lo[c];
        hi = a.f_hi[c];
        const uint32_t k = a.cut[c];
        const uint64_t n = hi - lo;
        if (n >= c_loc && k != 0) {   // n < c_loc: finished by local_root_kernel
            mid = lo + k;
            S = a.f_S[c];
            SL = a.cut_SL[c];
            Q = a.f_Q[c];
            uint64_t s_lo, s_mid;
            u128 q_lo, q_mid;
            pref12(a.PS1, a.PS2, a.t, lo, s_lo, q_lo);
            pref12(a.PS1, a.PS2, a.t, mid, s_mid, q_mid);
            QL = q_mid - q_lo;
            if (split_pays(n, S, Q, k, SL, QL, a.eps, a.z, a.k2, a.clamp)) {
                atomicOr(&a.flags[mid >> 5], 1u << (mid & 31));
                ntL = nontrivial(a.t, lo, mid);
                ntR = nontrivial(a.t, mid, hi);
            }
        }
    }
    // warp-aggregated append of (count << 32 | rows)
    const uint64_t mine = ((uint64_t)(ntL + ntR) << 32) | (uint64_t)((ntL ? mid - lo : 0u) + (ntR ? hi - mid : 0u));
    uint64_t incl = mine;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const uint64_t v = __shfl_up_sync(0xffffffffu, incl, o);
        if (lane >= o) incl += v;
    }
    uint64_t base = 0;
    const uint64_t wtot = __shfl_sync(0xffffffffu, incl, 31);
    if (lane == 31 && wtot) base = atomicAdd((unsigned long long *)a.total, (unsigned long long)wtot);
    base = __shfl_sync(0xffffffffu, base, 31);
    uint32_t idx = (uint32_t)((base + incl - mine) >> 32);
    SR_DCHECK(!(ntL || ntR) || idx + (ntL ? 1u : 0u) + (ntR ? 1u : 0u) <= 2u * (uint32_t)(*a.ctot >> 32));
    if (ntL) {
        a.nlo[idx] = lo; a.nhi[idx] = mid;
        a.nS[idx] = SL; a.nQ[idx] = QL;
        idx++;
    }
    if (ntR) {
        a.nlo[idx] = mid; a.nhi[idx] = hi;
        a.nS[idx] = S - SL; a.nQ[idx] = Q - QL;
    }
}

// ---------------------------------------------------------------- local subtrees
// One warp per frontier cluster of < local_rows() rows: cut (warp_best_cut),
// decision (split_pays, Q_L from the sampled prefix), then the children,
// depth first; the larger child waits on a per-warp stack and the smaller is
// processed next, so the stack holds at most log2(local_rows()) nodes.  Writes
// flags at the cuts; the cluster leaves the frontier.
constexpr int kLocalStack = 24;
struct LNode {
    uint64_t S;
    u128 Q;
    uint32_t lo, hi, depth, pad;
};

struct LocalArgs {
    const uint32_t *f_lo, *f_hi;
    const uint64_t *f_S;
    const u128 *f_Q;
    uint32_t C, level;
    const uint64_t *PS1;
    const u128 *PS2;
    const uint32_t *t, *TB;
    uint32_t *flags;   // leaf-start bitmap
    double eps, z, k2;
    int clamp;
    unsigned long long *rows;   // stats: rows scanned
    uint32_t *depth;            // stats: deepest level reached (1-based)
    uint32_t *err;
};

// warp: sum of t^2 over [x & ~31, x) (the partial chunk of a sampled prefix), all lanes
__device__ __forceinline__ u128 warp_partial_sq(const uint32_t *t, uint64_t x) {
    const int lane = threadIdx.x & 31;
    const uint64_t b = x & ~(kChunk - 1);
    uint64_t v = 0;
    if (b + lane < x) {
        const uint64_t tv = t[b + lane];
        v = tv * tv;
    }
    u128 s = v;
#pragma unroll
    for (int o = 16; o; o >>= 1) {
        const uint64_t lo_ = __shfl_xor_sync(0xffffffffu, (uint64_t)s, o);
        const uint64_t hi_ = __shfl_xor_sync(0xffffffffu, (uint64_t)(s >> 64), o);
        s += ((u128)hi_ << 64) | lo_;
    }
    return s;
}

__global__ void __launch_bounds__(256) local_root_kernel(LocalArgs a) {
    __shared__ LNode s_stack[8][kLocalStack];
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    const uint64_t nwarps = ((uint64_t)gridDim.x * blockDim.x) >> 5;
    uint64_t rows = 0;
    uint32_t dmax = 0;
    for (uint64_t c = ((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; c < a.C; c += nwarps) {
        LNode cur;
        cur.lo = a.f_lo[c];
        cur.hi = a.f_hi[c];
        if ((uint64_t)(cur.hi - cur.lo) >= c_loc) continue;
        cur.S = a.f_S[c];
        cur.Q = a.f_Q[c];
        cur.depth = a.level;
        int sp = 0;
        while (true) {   // cur is non-trivial
            const uint64_t n = cur.hi - cur.lo;
            if (cur.depth > a.level) rows += n;   // the frontier level counts the root node
            dmax = max(dmax, cur.depth + 1);
            const Cand b = warp_best_cut(a.t, a.PS1, a.TB, cur.lo, n, cur.S);
            bool have = false;
            LNode nx;
            if (b.k != 0) {
                const uint32_t mid = cur.lo + b.k;
                // Q_L = P2(mid) - P2(lo) from the sampled prefix (exact, mod 2^128)
                const u128 QL = (a.PS2[mid >> kChunkLog] + warp_partial_sq(a.t, mid)) -
                                (a.PS2[cur.lo >> kChunkLog] + warp_partial_sq(a.t, cur.lo));
                if (split_pays(n, cur.S, cur.Q, b.k, b.SL, QL, a.eps, a.z, a.k2, a.clamp)) {
                    if (lane == 0) atomicOr(&a.flags[mid >> 5], 1u << (mid & 31));
                    LNode L{b.SL, QL, cur.lo, mid, cur.depth + 1, 0};
                    LNode R{cur.S - b.SL, cur.Q - QL, mid, cur.hi, cur.depth + 1, 0};
                    const bool ntL = nontrivial(a.t, cur.lo, mid), ntR = nontrivial(a.t, mid, cur.hi);
                    if (ntL && ntR) {
                        const bool lbig = (mid - cur.lo) >= (cur.hi - mid);
                        if (sp == kLocalStack) {   // cannot happen: sizes halve along the stack
                            if (lane == 0) atomicOr(a.err, 4u);
                            break;
                        }
                        if (lane == 0) s_stack[w][sp] = lbig ? L : R;
                        sp++;
                        nx = lbig ? R : L;
                        have = true;
                    } else if (ntL) {
                        nx = L;
                        have = true;
                    } else if (ntR) {
                        nx = R;
                        have = true;
                    }
                }
            }
            if (!have) {
                if (sp == 0) break;
                __syncwarp();
                nx = s_stack[w][--sp];
            }
            __syncwarp();
            cur = nx;
        }
    }
    // stats (one atomic per warp)
    if (lane == 0 && rows) {
        atomicAdd(a.rows, (unsigned long long)rows);
        atomicMax(a.depth, dmax);
    }
}

// ---------------------------------------------------------------- frontier bookkeeping
__global__ void group_flags_kernel(const uint32_t *goff, uint32_t K, uint32_t *flags) {
    const uint64_t g = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (g < K && goff[g] < goff[g + 1]) atomicOr(&flags[goff[g] >> 5], 1u << (goff[g] & 31));
}


// leaf starts given from outside (multi-GPU: the leaves of a kernel split across
// ranks): entry i = (local kernel, rows from the kernel's local group start)
__global__ void fixed_flags_kernel(const uint32_t *cut, uint64_t m, const uint32_t *goff, uint32_t *flags) {
    const uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= m) return;
    const uint32_t p = goff[cut[2 * i]] + cut[2 * i + 1];
    atomicOr(&flags[p >> 5], 1u << (p & 31));
}

int stem_only_leaves(Ctx &c, uint64_t n, uint32_t K) {
    CK(cudaMemsetAsync(c.flags, 0, sizeof(uint32_t) * (n / 32 + 1), c.stream));
    group_flags_kernel<<<(unsigned)((K + 255) / 256), 256, 0, c.stream>>>(c.goff, K, c.flags);
    c.launches++;
    CK(cudaGetLastError());
    return STEM_OK;
}

static int ensure_frontier(Ctx &c, int b, uint64_t cap) {
    CKS(c.ensure(c.f_lo[b], c.cap_flo[b], sizeof(uint32_t) * cap));
    CKS(c.ensure(c.f_hi[b], c.cap_fhi[b], sizeof(uint32_t) * cap));
    CKS(c.ensure(c.f_S[b], c.cap_fS[b], sizeof(uint64_t) * cap));
    CKS(c.ensure(c.f_Q[b], c.cap_fQ[b], sizeof(u128) * cap));
    return STEM_OK;
}

int root_levels(Ctx &c, uint64_t n, uint32_t K, double eps, double z, double k2, int clamp, int split,
                uint64_t seed) {
    cudaStream_t st = c.stream;
    // the local subtree kernel implements the exact split only: the Lloyd rules
    // (split != 0) keep every cluster on the level path
    const uint64_t loc_rows = split != 0 ? 0 : local_rows();
    {
        const uint64_t b = big_rows();
        CK(cudaMemcpyToSymbolAsync(c_big, &b, sizeof(b), 0, cudaMemcpyHostToDevice, st));
        const uint64_t l = loc_rows < b ? loc_rows : b;
        CK(cudaMemcpyToSymbolAsync(c_loc, &l, sizeof(l), 0, cudaMemcpyHostToDevice, st));
        int b2 = 0;
        if (const char *e = getenv("STEMROOT_SPLIT_BOUND")) b2 = atoi(e) ? 1 : 0;
        CK(cudaMemcpyToSymbolAsync(c_bound2, &b2, sizeof(b2), 0, cudaMemcpyHostToDevice, st));
    }
    CKS(stem_only_leaves(c, n, K));
    // groups with many repeated times: their trees are built over values, beside the row levels
    DensePath dense{c};
    if (split == 0) CKS(dense.start(n, K, eps, z, k2, clamp));
    // initial frontier: non-trivial kernel groups, in kernel order, with exact S and Q
    {
        CKS(ensure_frontier(c, 0, (uint64_t)K + 1));
        CKS(c.ensure(c.scan_scratch, c.cap_scan, (scan_tiles(K) + 1) * sizeof(uint64_t)));
        const uint32_t *goff = c.goff, *t = c.t_sorted;
        const uint64_t *PS1 = c.PS1;
        const u128 *PS2 = c.PS2;
        uint32_t *nlo = c.f_lo[0], *nhi = c.f_hi[0];
        uint64_t *nS = c.f_S[0];
        u128 *nQ = c.f_Q[0];
        // skipped: kernels whose leaves are given (multi-GPU) or built on the value path
        const uint8_t *fixed = dense.on ? dense.sel_ : c.fixed_kernel;
        if (c.fixed_cuts && c.n_fixed_cuts) {
            fixed_flags_kernel<<<(unsigned)((c.n_fixed_cuts + 255) / 256), 256, 0, st>>>(c.fixed_cuts, c.n_fixed_cuts,
                                                                                      c.goff, c.flags);
            c.launches++;
        }
        const int tk = c.stage_begin("root_init");
        exclusive_scan<uint64_t>(
            [goff, t, fixed] __device__(uint64_t g) -> uint64_t {
                const uint32_t lo = goff[g], hi = goff[g + 1];
                return (nontrivial(t, lo, hi) && !(fixed && fixed[g])) ? ((1ull << 32) | (hi - lo)) : 0ull;
            },
            [nlo, nhi, nS, nQ, goff, t, PS1, PS2] __device__(uint64_t g, uint64_t pre, uint64_t v) {
                if (!v) return;
                const uint32_t idx = (uint32_t)(pre >> 32), lo = goff[g], hi = goff[g + 1];
                uint64_t s0, s1;
                u128 q0, q1;
                pref12(PS1, PS2, t, lo, s0, q0);
                pref12(PS1, PS2, t, hi, s1, q1);
                nlo[idx] = lo;
                nhi[idx] = hi;
                nS[idx] = s1 - s0;
                nQ[idx] = q1 - q0;
            },
            (uint64_t)K, (uint64_t *)c.scan_scratch, &c.scalars->ftot[0], st, &c.launches);
        c.stage_end(tk, 64 * (uint64_t)K);
        CK(cudaGetLastError());
    }
    // Levels, pipelined: level L+1 is enqueued before level L's frontier size is
    // known on the host.  Kernels read the size of the frontier they consume
    // from HBM (ftot[cur]); the host sizes grids and buffers from upper bounds
    // (a level at most doubles the cluster count and never adds rows) and reads
    // each level's exact total one level later (pinned ring + event), so the GPU
    // always has the next level queued.  The level after the last one runs on an
    // empty frontier (its kernels exit at once).  STEMROOT_LEVEL_SYNC=1, the
    // local-subtree option and STEMROOT_DEBUG_LEVELS use one host round trip per level.
    const bool pipelined = loc_rows == 0 && !debug_levels() &&
                           !(getenv("STEMROOT_LEVEL_SYNC") && getenv("STEMROOT_LEVEL_SYNC")[0] == '1');
    if (!c.h_lvl) {
        CK(cudaMallocHost((void **)&c.h_lvl, sizeof(uint64_t) * 4));
        for (int i = 0; i < 4; i++) CK(cudaEventCreateWithFlags(&c.ev_lvl[i], cudaEventDisableTiming));
    }
    uint64_t t0 = 0;
    CK(cudaMemcpyAsync(&t0, &c.scalars->ftot[0], sizeof(uint64_t), cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
    uint32_t levels = 0;
    // enqueue ROOT level `level` (1-based) consuming frontier cur, bounded by (Cub, Aub)
    const int ncm_l = split == 0 ? nc_mode() : -1;   // the exact rule's split kernels (read once per plan)
    auto enqueue_level = [&](uint32_t level, int cur, uint64_t Cub, uint64_t Aub) -> int {
        const int nxt = cur ^ 1;
        const uint64_t *ctot = &c.scalars->ftot[cur];
        uint64_t *ntot = &c.scalars->ftot[nxt];
        // Growing a buffer frees the old one, which the levels already queued
        // may still read (nxt is the input of the level queued before this
        // one): drain the stream first, then grow with 2x headroom so this
        // happens only O(log) times per ctx.
        const uint64_t max_ent = Aub / kBigSeg + Aub / big_rows() + 1;
        const bool grow = sizeof(uint32_t) * Cub > c.cap_cut || sizeof(uint64_t) * Cub > c.cap_cut_SL ||
                          sizeof(u128) * 2 * Cub > c.cap_fQ[nxt] ||
                          (split == 0 && (sizeof(BigEntry) * max_ent + sizeof(uint32_t) * (Cub + 1) > c.cap_big_ent ||
                                          sizeof(Cand) * max_ent > c.cap_big_part ||
                                          sizeof(unsigned long long) * Cub > c.cap_big_thr));
        if (grow) {
            CK(cudaStreamSynchronize(st));
            CKS(c.ensure(c.cut, c.cap_cut, 2 * sizeof(uint32_t) * Cub));
            CKS(c.ensure(c.cut_SL, c.cap_cut_SL, 2 * sizeof(uint64_t) * Cub));
            CKS(ensure_frontier(c, nxt, 4 * Cub));   // at most 2 children per cluster
            if (split == 0) {
                CKS(c.ensure(c.big_ent, c.cap_big_ent, 2 * (sizeof(BigEntry) * max_ent + sizeof(uint32_t) * (Cub + 1))));
                CKS(c.ensure(c.big_part, c.cap_big_part, 2 * sizeof(Cand) * max_ent));
                CKS(c.ensure(c.big_thr, c.cap_big_thr, 2 * sizeof(unsigned long long) * Cub));
            }
        }
        const int tk_l = loc_rows > 0 ? c.stage_begin("root_local") : -1;
        if (loc_rows > 0) {
            LocalArgs la{c.f_lo[cur], c.f_hi[cur], c.f_S[cur], c.f_Q[cur], (uint32_t)Cub, level - 1, c.PS1, c.PS2,
                         c.t_sorted, c.TB, c.flags, eps, z, k2, clamp, &c.scalars->local_rows, &c.scalars->local_depth,
                         &c.scalars->err};
            const uint64_t blocks = (Cub + 7) / 8;
            local_root_kernel<<<(unsigned)min(blocks, (uint64_t)c.sms * 64), 256, 0, st>>>(la);
            c.launches++;
        }
        if (tk_l >= 0) c.stage_end(tk_l, 4 * Aub);
        CK(cudaGetLastError());
        const int tk_s = c.stage_begin("root_split");
        if (split != 0) {   // Lloyd variants: one warp per cluster, every size
            const unsigned g = (unsigned)min((Cub + 7) / 8, (uint64_t)c.sms * 16);
            const uint32_t k0 = (uint32_t)seed, k1 = (uint32_t)(seed >> 32);
            uint32_t *q = &c.scalars->nc_queue[level & 1];
            CK(cudaMemsetAsync(q, 0, sizeof(uint32_t), st));
            if (split == 2)
                lloyd_split_kernel<true><<<g, 256, 0, st>>>(c.f_lo[cur], c.f_hi[cur], c.f_S[cur], c.f_Q[cur], ctot,
                                                            c.t_sorted, c.PS1, c.PS2, k0, k1, c.cut, c.cut_SL, q);
            else
                lloyd_split_kernel<false><<<g, 256, 0, st>>>(c.f_lo[cur], c.f_hi[cur], c.f_S[cur], c.f_Q[cur], ctot,
                                                             c.t_sorted, c.PS1, c.PS2, k0, k1, c.cut, c.cut_SL, q);
            c.launches++;
        } else {
        // the small-cluster warps run on a side stream beside the big-cluster
        // chain (both latency-bound; they read the same frontier and write
        // disjoint cuts), joined before the decision
        if (!c.side) {
            CK(cudaStreamCreateWithFlags(&c.side, cudaStreamNonBlocking));
            CK(cudaEventCreateWithFlags(&c.ev_fork, cudaEventDisableTiming));
            CK(cudaEventCreateWithFlags(&c.ev_join, cudaEventDisableTiming));
        }
        const bool overlap = split_overlap();
        cudaStream_t sst = overlap ? c.side : st;
        if (overlap) {
            CK(cudaEventRecord(c.ev_fork, st));
            CK(cudaStreamWaitEvent(c.side, c.ev_fork, 0));
        }
        const int ncm = ncm_l;
        uint32_t *q_cur = &c.scalars->nc_queue[level & 1], *q_next = &c.scalars->nc_queue[(level + 1) & 1];
        if (ncm == 1 || (ncm == 2 && level == 1)) CK(cudaMemsetAsync(q_cur, 0, sizeof(uint32_t), st));
        if (ncm == 2) {   // every cluster by the nearest-centre descent
            constexpr uint64_t wpb = SR_NC_THREADS / 32;
            const uint64_t blocks = (Cub + wpb - 1) / wpb;
            nc_split_kernel<<<(unsigned)min(blocks, (uint64_t)c.sms * 16 * (8 / wpb)), SR_NC_THREADS, 0, st>>>(
                c.f_lo[cur], c.f_hi[cur], c.f_S[cur], ctot, c.t_sorted, c.PS1, c.TB, c.cut, c.cut_SL, 0,
                NcStats{&c.scalars->split_chunks, &c.scalars->split_scanned}, q_cur, q_next, ntot);
            c.launches++;
        } else {
        if (loc_rows < big_rows()) {
            const uint64_t blocks = (Cub + 7) / 8;
            static int minb = -1;   // STEMROOT_SMALL_MINB: resident blocks per SM the registers are sized for
            if (minb < 0) minb = getenv("STEMROOT_SMALL_MINB") ? atoi(getenv("STEMROOT_SMALL_MINB")) : 4;
            if (minb == 3)
                small_split_kernel<3><<<(unsigned)min(blocks, (uint64_t)c.sms * 16), 256, 0, sst>>>(
                    c.f_lo[cur], c.f_hi[cur], c.f_S[cur], ctot, c.t_sorted, c.PS1, c.TB, c.cut, c.cut_SL);
            else
                small_split_kernel<4><<<(unsigned)min(blocks, (uint64_t)c.sms * 16), 256, 0, sst>>>(
                    c.f_lo[cur], c.f_hi[cur], c.f_S[cur], ctot, c.t_sorted, c.PS1, c.TB, c.cut, c.cut_SL);
            c.launches++;
        }
        if (ncm == 1) {   // big clusters by the nearest-centre descent, beside the small-cluster warps
            constexpr uint64_t wpb = SR_NC_THREADS / 32;
            const uint64_t blocks = (Cub + wpb - 1) / wpb;
            nc_split_kernel<<<(unsigned)min(blocks, (uint64_t)c.sms * 16 * (8 / wpb)), SR_NC_THREADS, 0, st>>>(
                c.f_lo[cur], c.f_hi[cur], c.f_S[cur], ctot, c.t_sorted, c.PS1, c.TB, c.cut, c.cut_SL, big_rows(),
                NcStats{&c.scalars->split_chunks, &c.scalars->split_scanned}, q_cur, nullptr, nullptr);
            c.launches++;
        } else {
        // big clusters: entries (cluster, segment), chunk-bound argmax, per-cluster reduce
        BigEntry *ent = (BigEntry *)c.big_ent;
        uint32_t *first_ent = (uint32_t *)(ent + max_ent);
        CK(cudaMemsetAsync(&c.scalars->big_count, 0, sizeof(uint32_t), st));
        big_entries_kernel<<<(unsigned)((Cub + 255) / 256), 256, 0, st>>>(c.f_lo[cur], c.f_hi[cur], ctot, ent, first_ent,
                                                                         &c.scalars->big_count,
                                                                         (unsigned long long *)c.big_thr);
        BigArgs ba{ent, &c.scalars->big_count, c.f_lo[cur], c.f_hi[cur], c.f_S[cur], c.PS1, c.t_sorted, c.TB,
                   (unsigned long long *)c.big_thr, (Cand *)c.big_part, &c.scalars->split_chunks,
                   &c.scalars->split_scanned};
        if (seed_on()) {
            big_seed_kernel<<<(unsigned)min((max_ent + 7) / 8, (uint64_t)c.sms * 8), 256, 0, st>>>(ba);
            c.launches++;
        }
        static const cudaError_t big_attr =
            cudaFuncSetAttribute(big_split_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kBigSmem);
        CK(big_attr);
        big_split_kernel<<<(unsigned)min(max_ent, (uint64_t)c.sms * 8), kBigThreads, kBigSmem, st>>>(ba);
        c.launches += 2;
        big_reduce_kernel<<<(unsigned)min(Cub, (uint64_t)4096), 32, 0, st>>>(c.f_lo[cur], c.f_hi[cur], ctot, first_ent,
                                                                        (const Cand *)c.big_part, c.cut, c.cut_SL);
        c.launches += 2;
        }   // ncm != 1
        if (overlap) {
            CK(cudaEventRecord(c.ev_join, c.side));
            CK(cudaStreamWaitEvent(st, c.ev_join, 0));
        }
        }   // ncm != 2
        }   // split == 0
        c.stage_end(tk_s, 4 * Aub + 20 * Cub);
        CK(cudaGetLastError());
        const int tk_d = c.stage_begin("root_decide");
        if (ncm_l != 2) CK(cudaMemsetAsync(ntot, 0, sizeof(uint64_t), st));   // else zeroed by nc_split
        DecideArgs da{c.f_lo[cur], c.f_hi[cur], c.cut, c.f_S[cur], c.cut_SL, c.f_Q[cur], ctot, c.PS1, c.PS2,
                      c.t_sorted, c.flags, c.f_lo[nxt], c.f_hi[nxt], c.f_S[nxt], c.f_Q[nxt],
                      ntot, eps, z, k2, clamp};
        decide_kernel<<<(unsigned)((Cub + 255) / 256), 256, 0, st>>>(da);
        c.launches += 1;
        c.stage_end(tk_d, 96 * Cub);
        CK(cudaGetLastError());
        if (debug_levels()) {   // STEMROOT_DEBUG_LEVELS=1: per-level frontier and big-path stats on stderr
            DevScalars hs;
            CK(cudaMemcpyAsync(&hs, c.scalars, sizeof(DevScalars), cudaMemcpyDeviceToHost, st));
            CK(cudaStreamSynchronize(st));
            fprintf(stderr, "level %u: clusters %llu rows %llu big_entries %u chunks %llu scanned %llu\n", level,
                    (unsigned long long)(hs.ftot[cur] >> 32), (unsigned long long)(hs.ftot[cur] & 0xFFFFFFFFull),
                    hs.big_count, hs.split_chunks, hs.split_scanned);
        }
        CK(cudaMemcpyAsync(&c.h_lvl[level & 3], ntot, sizeof(uint64_t), cudaMemcpyDeviceToHost, st));
        CK(cudaEventRecord(c.ev_lvl[level & 3], st));
        return STEM_OK;
    };
    uint64_t Cprev = t0 >> 32, Aprev = t0 & 0xFFFFFFFFull;   // the frontier level 1 consumes (exact)
    if (Cprev > 0) {
        if (!pipelined) {
            int cur = 0;
            for (uint32_t level = 1; Cprev > 0; level++) {
                levels = level;
                c.stats.active_rows += Aprev;
                CKS(enqueue_level(level, cur, Cprev, Aprev));
                CKS(dense.pump());
                CK(cudaEventSynchronize(c.ev_lvl[level & 3]));
                Cprev = c.h_lvl[level & 3] >> 32;
                Aprev = c.h_lvl[level & 3] & 0xFFFFFFFFull;
                cur ^= 1;
            }
        } else {
            // level 1 with the exact bound, then level L+1 queued while level L runs
            CKS(enqueue_level(1, 0, Cprev, Aprev));
            uint64_t Cl = Cprev, Al = Aprev;   // exact size of the frontier level `level` consumes
            for (uint32_t level = 1;; level++) {
                levels = level;
                c.stats.active_rows += Al;
                // level + 1 consumes level's output: at most 2 Cl clusters, Al rows
                CKS(enqueue_level(level + 1, level & 1, 2 * Cl, Al));
                CKS(dense.pump());
                CK(cudaEventSynchronize(c.ev_lvl[level & 3]));
                Cl = c.h_lvl[level & 3] >> 32;
                Al = c.h_lvl[level & 3] & 0xFFFFFFFFull;
                if (Cl == 0) break;   // the queued level runs on an empty frontier
            }
        }
    }
    CKS(dense.finish(c.flags));
    DevScalars hs;
    CK(cudaMemcpyAsync(&hs, c.scalars, sizeof(DevScalars), cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
    if (hs.err & 4u) return STEM_E_CUDA;   // local stack overflow (unreachable)
    c.stats.levels = levels > hs.local_depth ? levels : hs.local_depth;
    c.stats.active_rows += hs.local_rows;
    c.stats.split_chunks = hs.split_chunks;
    c.stats.split_scanned = hs.split_scanned;
    return STEM_OK;
}


// ---------------------------------------------------------------- ROOT over a value histogram
// ROOT's decisions depend only on the multiset of a cluster's times: a cut
// lies between two distinct values, D_k = n S_L - S k and the Eq. 7/8 test use
// the counts and sums below it.  So the tree of a kernel can be built from its
// distinct values and their counts alone -- exactly the tree the row levels
// build.  Two users: the single-GPU plan hands kernels with many repeated
// times (C5's large kernels: 532 M rows, 23.5 M distinct values) to this path,
// which scans values instead of rows; the multi-GPU plan builds the tree of a
// kernel larger than a rank's share from the merged histogram (dist.cu).
//
// A value u (interior of its group) is described by kc[u], the rows before it
// (dense path: its first row; histogram: the prefix count), Ps[u], the sum of
// t before it, and the sum of t^2 before it (histogram: Pq[u]; dense path:
// from the row prefix PS2 at that row, needed only at accepted cuts).  A
// cluster carries its value range, rows, and exact S, Q (and the prefixes at
// its start), like the row frontier.  Levels are pipelined like the row
// levels: every kernel reads the size of the frontier it consumes from device
// memory, the grids are persistent, and the host learns a level's output size
// later (pinned ring + events), so the run can advance on a side stream from
// the row loop without blocking it (VrRun::pump).
struct VH {
    uint64_t c, s;
    u128 q;
};
__host__ __device__ __forceinline__ VH operator+(const VH &a, const VH &b) { return VH{a.c + b.c, a.s + b.s, a.q + b.q}; }
__host__ __device__ __forceinline__ VH operator-(const VH &a, const VH &b) { return VH{a.c - b.c, a.s - b.s, a.q - b.q}; }

constexpr uint32_t kVrEV = 1024;                 // values per entry (one warp)
constexpr unsigned long long kVrMask = (1ull << 40) - 1;
constexpr int kVrRing = 8;

struct VrClu {          // a frontier cluster
    uint32_t lo, hi;    // value range [lo, hi)
    uint32_t k0, n;     // rows before it (kc at lo), its rows
    uint64_t s0, S;     // sum t before it, its sum
    u128 q0, Q;         // sum t^2 before it, its sum
    uint32_t ef, pad;   // first entry
};

struct VrDev {
    const uint32_t *kc;                          // [D] rows before value u
    const uint64_t *Ps;                          // [D] sum t before value u
    const u128 *Pq;                              // [D] sum t^2 before value u (nullptr: from the rows)
    const uint64_t *PS1;                         // dense path: row prefixes and times
    const u128 *PS2;
    const uint32_t *t;
    VrClu *clu[2];                               // frontier f
    uint32_t *eclu, *ea, *eb;                    // entries of the level being cut
    Cand *cand;                                  // best cut per entry
    unsigned long long *cnt;                     // [2] (clusters << 40) | entries, per frontier
    unsigned long long *active;                  // rows of the clusters decided (ROOT active rows)
    uint8_t *vflag;                              // 1 at the first value of every leaf
    double eps, z, k2;
    int clamp;
};

static VrDev &vdev(VrRun &r) {
    static_assert(sizeof(VrDev) <= sizeof(r.devs.b), "VrRun::devs too small");
    return *reinterpret_cast<VrDev *>(r.devs.b);
}

__device__ __forceinline__ uint32_t vr_nent(uint32_t nv) { return (nv + kVrEV - 1) / kVrEV; }

__device__ __forceinline__ u128 vr_q(const VrDev &a, uint32_t u) {
    if (a.Pq) return a.Pq[u];
    uint64_t s;
    u128 q;
    pref12(a.PS1, a.PS2, a.t, a.kc[u], s, q);
    return q;
}

__device__ __forceinline__ void vr_push(const VrDev &a, int f, const VrClu &x) {
    const unsigned long long p = atomicAdd(&a.cnt[f], (1ull << 40) | vr_nent(x.hi - x.lo));
    VrClu y = x;
    y.ef = (uint32_t)(p & kVrMask);
    a.clu[f][p >> 40] = y;
}

// first frontier from prefix arrays over [0, D] (histogram input)
__global__ void vr_init_hist_kernel(VrDev a, const uint32_t *goffv, uint32_t G) {
    const uint32_t g = blockIdx.x * blockDim.x + threadIdx.x;
    if (g >= G) return;
    const uint32_t v0 = goffv[g], v1 = goffv[g + 1];
    if (v1 > v0) a.vflag[v0] = 1;
    if (v1 - v0 < 2) return;   // at least two distinct values
    VrClu x{};
    x.lo = v0;
    x.hi = v1;
    x.k0 = a.kc[v0];
    x.n = a.kc[v1] - x.k0;
    x.s0 = a.Ps[v0];
    x.S = a.Ps[v1] - x.s0;
    x.q0 = a.Pq[v0];
    x.Q = a.Pq[v1] - x.q0;
    vr_push(a, 0, x);
}

// first frontier of the dense groups: rows and moments from the row prefixes
__global__ void vr_init_rows_kernel(VrDev a, const uint32_t *goffv, const uint32_t *dgrp, uint32_t G,
                                    const uint32_t *goff) {
    const uint32_t j = blockIdx.x * blockDim.x + threadIdx.x;
    if (j >= G) return;
    const uint32_t v0 = goffv[j], v1 = goffv[j + 1], g = dgrp[j];
    if (v1 > v0) a.vflag[v0] = 1;
    if (v1 - v0 < 2) return;
    VrClu x{};
    x.lo = v0;
    x.hi = v1;
    x.k0 = goff[g];
    x.n = goff[g + 1] - goff[g];
    uint64_t s1;
    u128 q1;
    pref12(a.PS1, a.PS2, a.t, goff[g], x.s0, x.q0);
    pref12(a.PS1, a.PS2, a.t, goff[g + 1], s1, q1);
    x.S = s1 - x.s0;
    x.Q = q1 - x.q0;
    vr_push(a, 0, x);
}

// one warp per cluster of frontier f: its entry records
__global__ void vr_expand_kernel(VrDev a, int f) {
    const uint64_t C = a.cnt[f] >> 40;
    const int lane = threadIdx.x & 31;
    const uint64_t nw = (uint64_t)gridDim.x * (blockDim.x >> 5);
    for (uint64_t ci = (uint64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); ci < C; ci += nw) {
        const uint32_t lo = a.clu[f][ci].lo, hi = a.clu[f][ci].hi, e0 = a.clu[f][ci].ef, ne = vr_nent(hi - lo);
        for (uint32_t j = lane; j < ne; j += 32) {
            a.eclu[e0 + j] = (uint32_t)ci;
            a.ea[e0 + j] = lo + j * kVrEV;
            a.eb[e0 + j] = min(lo + (j + 1) * kVrEV, hi);
        }
    }
}

// one warp per entry: the exact best cut over its distinct-value boundaries
// u (left = values [lo, u)), eval_cut as on the row path
__global__ void __launch_bounds__(256) vr_cut_kernel(VrDev a, int f) {
    const uint64_t E = a.cnt[f] & kVrMask;
    const int lane = threadIdx.x & 31;
    const uint64_t nw = (uint64_t)gridDim.x * (blockDim.x >> 5);
    for (uint64_t e = (uint64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); e < E; e += nw) {
        const VrClu &x = a.clu[f][a.eclu[e]];
        const uint32_t k0 = x.k0, n = x.n, ua = max(a.ea[e], x.lo + 1), ub = a.eb[e];
        const uint64_t s0 = x.s0, S = x.S;
        Cand best = no_cand();
        for (uint32_t b0 = ua; b0 < ub; b0 += 8 * 32) {   // 8 loads in flight per lane, then the scores
            uint32_t kk[8];
            uint64_t ss[8];
#pragma unroll
            for (int q = 0; q < 8; q++) {
                const uint32_t u = b0 + lane + 32 * q;
                kk[q] = u < ub ? a.kc[u] : 0u;
                ss[q] = u < ub ? a.Ps[u] : 0ull;
            }
#pragma unroll 1
            for (int q = 0; q < 8; q++)
                if (b0 + lane + 32 * q < ub) eval_cut(kk[q] - k0, n, S, ss[q] - s0, best);
        }
#pragma unroll 1
        for (int o = 16; o; o >>= 1) {
            const Cand v = shfl_cand_xor(best, o);
            if (better(v, best)) best = v;
        }
        if (lane == 0) a.cand[e] = best;
    }
}

// one warp per cluster: the best of its entries, the Eq. 7/8 decision, the children
__global__ void __launch_bounds__(256) vr_decide_kernel(VrDev a, int f) {
    const uint64_t C = a.cnt[f] >> 40;
    const int lane = threadIdx.x & 31;
    const uint64_t nw = (uint64_t)gridDim.x * (blockDim.x >> 5);
    for (uint64_t ci = (uint64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); ci < C; ci += nw) {
        const VrClu x = a.clu[f][ci];
        const uint32_t ne = vr_nent(x.hi - x.lo);
        Cand best = no_cand();
        for (uint32_t j = lane; j < ne; j += 32) {
            const Cand v = a.cand[x.ef + j];
            if (better(v, best)) best = v;
        }
#pragma unroll 1
        for (int o = 16; o; o >>= 1) {
            const Cand v = shfl_cand_xor(best, o);
            if (better(v, best)) best = v;
        }
        if (lane != 0) continue;
        atomicAdd(a.active, (unsigned long long)x.n);
        if (!best.k) continue;
        uint32_t l = x.lo + 1, h = x.hi;   // the value index with best.k rows before it
        while (l < h) {
            const uint32_t mid = l + (h - l) / 2;
            if (a.kc[mid] - x.k0 < best.k) l = mid + 1; else h = mid;
        }
        const uint32_t u = l;
        const u128 QL = vr_q(a, u) - x.q0;
        if (!split_pays(x.n, x.S, x.Q, best.k, best.SL, QL, a.eps, a.z, a.k2, a.clamp)) continue;
        a.vflag[u] = 1;
        if (u - x.lo >= 2) {
            VrClu L = x;
            L.hi = u;
            L.n = best.k;
            L.S = best.SL;
            L.Q = QL;
            vr_push(a, f ^ 1, L);
        }
        if (x.hi - u >= 2) {
            VrClu R = x;
            R.lo = u;
            R.k0 = x.k0 + best.k;
            R.n = x.n - best.k;
            R.s0 = x.s0 + best.SL;
            R.S = x.S - best.SL;
            R.q0 = x.q0 + QL;
            R.Q = x.Q - QL;
            vr_push(a, f ^ 1, R);
        }
    }
}

size_t vr_work_bytes(uint64_t D) {
    const uint64_t Ccap = D / 2 + 2, Ecap = Ccap + D / kVrEV + 2;
    return 16 * 8 + 2 * sizeof(VrClu) * Ccap + sizeof(uint32_t) * 3 * Ecap + sizeof(Cand) * Ecap + 512;
}

// Lays out one run in c.vr_work (sized by the caller with vr_work_bytes(D)).
int VrRun::setup(const VrSource &src, uint64_t Dv, double eps, double z, double k2, int clamp, uint8_t *vflag,
                 cudaStream_t s) {
    st = s;
    D = Dv;
    enq = done = 0;
    finished = false;
    const uint64_t Ccap = D / 2 + 2, Ecap = Ccap + D / kVrEV + 2;
    VrDev d{};
    d.kc = src.kc;
    d.Ps = src.Ps;
    d.Pq = src.Pq;
    d.PS1 = c.PS1;
    d.PS2 = c.PS2;
    d.t = c.t_sorted;
    char *w = (char *)c.vr_work;
    auto take = [&](size_t bytes) {
        char *p = w;
        w += (bytes + 15) & ~(size_t)15;
        return (void *)p;
    };
    d.cnt = (unsigned long long *)take(16 * 8);
    d.active = d.cnt + 2;
    for (int f = 0; f < 2; f++) d.clu[f] = (VrClu *)take(sizeof(VrClu) * Ccap);
    d.eclu = (uint32_t *)take(sizeof(uint32_t) * Ecap);
    d.ea = (uint32_t *)take(sizeof(uint32_t) * Ecap);
    d.eb = (uint32_t *)take(sizeof(uint32_t) * Ecap);
    d.cand = (Cand *)take(sizeof(Cand) * Ecap);
    d.vflag = vflag;
    d.eps = eps;
    d.z = z;
    d.k2 = k2;
    d.clamp = clamp;
    vdev(*this) = d;
    if (!c.h_vr) {
        CK(cudaMallocHost((void **)&c.h_vr, sizeof(uint64_t) * (kVrRing + 1)));
        for (int i = 0; i < kVrRing; i++) CK(cudaEventCreateWithFlags(&c.ev_vr[i], cudaEventDisableTiming));
    }
    CK(cudaMemsetAsync(d.cnt, 0, 16 * 8, st));
    CK(cudaMemsetAsync(vflag, 0, D + 1, st));
    if (src.G) {
        if (src.dgrp)
            vr_init_rows_kernel<<<(src.G + 255) / 256, 256, 0, st>>>(d, src.goffv, src.dgrp, src.G, src.goff);
        else
            vr_init_hist_kernel<<<(src.G + 255) / 256, 256, 0, st>>>(d, src.goffv, src.G);
        launches++;
    }
    CK(cudaGetLastError());
    return STEM_OK;
}

int VrRun::enqueue_one() {
    const int f = (int)(enq & 1);
    const unsigned g = (unsigned)c.sms * 8;
    const VrDev &dev = vdev(*this);
    vr_expand_kernel<<<g, 256, 0, st>>>(dev, f);
    vr_cut_kernel<<<g, 256, 0, st>>>(dev, f);
    CK(cudaMemsetAsync(&dev.cnt[f ^ 1], 0, sizeof(unsigned long long), st));
    vr_decide_kernel<<<g, 256, 0, st>>>(dev, f);
    launches += 3;
    const int r = (int)(enq % kVrRing);
    CK(cudaMemcpyAsync(&c.h_vr[r], &dev.cnt[f ^ 1], sizeof(uint64_t), cudaMemcpyDeviceToHost, st));
    CK(cudaEventRecord(c.ev_vr[r], st));
    CK(cudaGetLastError());
    enq++;
    return STEM_OK;
}

// Advances the run: reads finished levels, keeps up to 3 levels queued.
// block = false never waits on the GPU (called from the row loop).
int VrRun::pump(bool block) {
    while (!finished) {
        while (done < enq) {
            const int r = (int)(done % kVrRing);
            if (block) {
                CK(cudaEventSynchronize(c.ev_vr[r]));
            } else {
                const cudaError_t q = cudaEventQuery(c.ev_vr[r]);
                if (q == cudaErrorNotReady) {
                    (void)cudaGetLastError();
                    break;
                }
                CK(q);
            }
            done++;
            if ((c.h_vr[r] >> 40) == 0) {   // no cluster left: the levels queued after it are empty
                finished = true;
                break;
            }
        }
        if (finished) break;
        if (enq - done < 3) CKS(enqueue_one());
        else if (!block) break;
    }
    return STEM_OK;
}

int VrRun::finish(uint64_t *active_rows) {
    CKS(pump(true));
    uint64_t act = 0;
    CK(cudaMemcpyAsync(&act, vdev(*this).active, sizeof(uint64_t), cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
    if (active_rows) *active_rows = act;
    levels = (uint32_t)done;
    return STEM_OK;
}

int root_values(Ctx &c, const uint32_t *vt, const uint64_t *vcnt, const uint32_t *goffv, uint32_t G, uint64_t D,
                double eps, double z, double k2, int clamp, uint8_t *vflag) {
    cudaStream_t st = c.stream;
    // prefix arrays over the values (D + 1 entries: the last is the total)
    CKS(c.ensure(c.vr_P, c.cap_vr_P, (sizeof(uint32_t) + sizeof(uint64_t) + sizeof(u128)) * (D + 2) + 64 +
                                     (scan_tiles(D + 1) + 2) * sizeof(VH)));
    u128 *Pq = (u128 *)c.vr_P;
    uint64_t *Ps = (uint64_t *)(Pq + (D + 2));
    uint32_t *Pc = (uint32_t *)(Ps + (D + 2));
    VH *scratch = (VH *)(((uintptr_t)(Pc + (D + 2)) + 63) & ~(uintptr_t)63);
    CKS(c.ensure(c.vr_work, c.cap_vr_work, vr_work_bytes(D)));
    exclusive_scan<VH>(
        [vt, vcnt, D] __device__(uint64_t u) -> VH {
            if (u >= D) return VH{0, 0, 0};
            const uint64_t cn = vcnt[u], tv = vt[u];
            return VH{cn, cn * tv, (u128)cn * ((u128)tv * tv)};
        },
        [Pc, Ps, Pq] __device__(uint64_t u, VH pre, VH) {
            Pc[u] = (uint32_t)pre.c;
            Ps[u] = pre.s;
            Pq[u] = pre.q;
        },
        D + 1, scratch, (VH *)c.scalars->wide_total, st, &c.launches);
    VrRun run{c};
    VrSource src{};
    src.kc = Pc;
    src.Ps = Ps;
    src.Pq = Pq;
    src.goffv = goffv;
    src.G = G;
    CKS(run.setup(src, D, eps, z, k2, clamp, vflag, st));
    CKS(run.finish(nullptr));
    c.launches += run.launches;
    return STEM_OK;
}

// ---------------------------------------------------------------- kernels with many repeated times
// A kernel group of >= STEMROOT_VALUE_ROWS rows (default 0 = off; 2^18 was the round-2 default) whose
// times repeat (a 1024-point sample finds t[i] == t[i-1] at >= 1 - 1/R of the
// points, R = STEMROOT_VALUE_RATIO, default 4) is handed to the value path:
// its distinct values are listed once (first row, sum of t before it), its
// tree is built by VrRun on a side stream while the row levels handle the
// other groups, and its leaf starts are set in the row flags.  The tree is the
// one the row levels would build (same cuts, same decisions), so this only
// changes the cost: C5's 79 largest kernels hold 53 % of the rows but 2.4 % of
// the distinct values.  Off by default since the nearest-centre descent: the
// row levels then decide those groups in less time than this path's listing.
constexpr uint32_t kWinRows = 2048;   // one warp's window of a dense group (64 aligned 32-row chunks)

static uint32_t value_rows() {   // read per plan (tests switch it)
    const char *e = getenv("STEMROOT_VALUE_ROWS");
    // default 0 (off): with the nearest-centre descent the row levels decide such
    // groups faster than the value path's own preparation (C5: 31.7 vs 33.0 ms per plan)
    const long v = e ? atol(e) : 0;
    return v < 0 ? 0u : (uint32_t)v;
}

static uint32_t value_ratio() {
    const char *e = getenv("STEMROOT_VALUE_RATIO");
    const long v = e ? atol(e) : 4;
    return v < 2 ? 2u : (uint32_t)v;
}

// one warp per group: sel[g] = 1 fixed (given leaves), 2 dense, 0 row path
__global__ void dense_select_kernel(const uint32_t *goff, const uint32_t *t, uint32_t K, const uint8_t *fixed,
                                    uint32_t min_rows, uint32_t ratio, uint8_t *sel, unsigned long long *acc) {
    const uint32_t g = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int lane = threadIdx.x & 31;
    if (g >= K) return;
    const uint32_t lo = goff[g], n = goff[g + 1] - lo;
    uint8_t v = fixed && fixed[g] ? 1 : 0;
    if (!v && min_rows && n >= min_rows && n >= 2) {
        uint32_t rep = 0;
        for (uint32_t j = lane; j < 1024; j += 32) {
            const uint32_t i = lo + 1 + (uint32_t)(((uint64_t)j * (n - 1)) >> 10);
            rep += t[i] == t[i - 1];
        }
        for (int o = 16; o; o >>= 1) rep += __shfl_xor_sync(0xffffffffu, rep, o);
        if ((uint64_t)rep * ratio >= 1024ull * (ratio - 1)) v = 2;
    }
    if (lane == 0) {
        sel[g] = v;
        if (v == 2) {
            atomicAdd(&acc[0], 1ull);
            atomicAdd(&acc[1], (unsigned long long)((n + (lo & 31u) + kWinRows - 1) / kWinRows));
        }
    }
}

struct DenseWin {   // window w of the dense groups -> group rows [glo, ghi), window rows [a, b), a 32-aligned
    const uint32_t *dgrp, *dwinf, *goff;
    uint32_t Gd;
    __device__ void operator()(uint32_t w, uint32_t &glo, uint32_t &ghi, uint32_t &a, uint32_t &b) const {
        const uint32_t j = (uint32_t)upper_bound(dwinf, (uint64_t)Gd + 1, w) - 1, g = dgrp[j];
        glo = goff[g];
        ghi = goff[g + 1];
        a = (glo & ~31u) + (w - dwinf[j]) * kWinRows;
        b = min(a + kWinRows, ghi);
    }
};

// Value starts among the rows [c, c + 128) of a window, 4 per lane (c is
// 32-aligned, so the uint4 loads are aligned; t_sorted has 4 rows of slack):
// bit r of the result = row c + 4 lane + r starts a value of the group.
// v = the 4 times (0 where the lane's first row is at or after b).
__device__ __forceinline__ uint32_t win_starts4(uint4 v, uint32_t c, uint32_t glo, uint32_t b, uint32_t tprev) {
    const int lane = threadIdx.x & 31;
    const uint32_t i0 = c + 4 * lane;
    uint32_t prev = __shfl_up_sync(0xffffffffu, v.w, 1);
    if (lane == 0) prev = tprev;   // t[c - 1] (any value when c <= glo)
    const uint32_t e[4] = {v.x, v.y, v.z, v.w};
    uint32_t f = 0;
#pragma unroll
    for (int r = 0; r < 4; r++) {
        const uint32_t i = i0 + r;
        const uint32_t p = r ? e[r - 1] : prev;
        if (i >= glo && i < b && (i == glo || e[r] != p)) f |= 1u << r;
    }
    return f;
}

__device__ __forceinline__ uint4 win_load(const uint32_t *t, uint32_t c, uint32_t b) {
    const uint32_t i0 = c + 4 * (threadIdx.x & 31);
    return i0 < b ? *reinterpret_cast<const uint4 *>(t + i0) : make_uint4(0, 0, 0, 0);
}

// one warp per window: distinct values (value starts) in it
__global__ void __launch_bounds__(256) dense_count_kernel(DenseWin dw, const uint32_t *t, uint32_t NW,
                                                          uint32_t *wcnt) {
    const int lane = threadIdx.x & 31;
    const uint32_t nw = gridDim.x * (blockDim.x >> 5);
    for (uint32_t w = blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); w < NW; w += nw) {
        uint32_t glo, ghi, a, b;
        dw(w, glo, ghi, a, b);
        uint32_t cnt = 0;
        uint32_t tprev = a > glo ? t[a - 1] : 0u;
        uint4 v = win_load(t, a, b);
        for (uint32_t c = a; c < b; c += 128) {
            const uint4 vn = c + 128 < b ? win_load(t, c + 128, b) : make_uint4(0, 0, 0, 0);   // next, in flight
            cnt += __popc(win_starts4(v, c, glo, b, tprev));
            tprev = __shfl_sync(0xffffffffu, v.w, 31);
            v = vn;
        }
        for (int o = 16; o; o >>= 1) cnt += __shfl_xor_sync(0xffffffffu, cnt, o);
        if (lane == 0) wcnt[w] = cnt;
    }
}

// one warp per window: the value list in row order, vpos[u] = first row of
// value u, Ps[u] = sum of t before it (PS1 at the 32-row chunk c + a warp scan)
__global__ void __launch_bounds__(256) dense_write_kernel(DenseWin dw, const uint32_t *t, const uint64_t *PS1,
                                                          uint32_t NW, const uint32_t *woff, uint32_t *vpos,
                                                          uint64_t *Ps) {
    const int lane = threadIdx.x & 31;
    const uint32_t nw = gridDim.x * (blockDim.x >> 5);
    for (uint32_t w = blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); w < NW; w += nw) {
        uint32_t glo, ghi, a, b;
        dw(w, glo, ghi, a, b);
        uint32_t off = woff[w];
        uint32_t tprev = a > glo ? t[a - 1] : 0u;
        uint4 v = win_load(t, a, b);
        for (uint32_t c = a; c < b; c += 128) {
            const uint4 vn = c + 128 < b ? win_load(t, c + 128, b) : make_uint4(0, 0, 0, 0);   // next, in flight
            const uint32_t f = win_starts4(v, c, glo, b, tprev);
            tprev = __shfl_sync(0xffffffffu, v.w, 31);
            const uint4 vc = v;
            v = vn;
            const uint32_t nf = __popc(f);
            if (!__any_sync(0xffffffffu, nf != 0)) continue;
            // Ps: rows of [c, c + 128) before i, whatever their group (PS1 is the global prefix;
            // v holds every row below b, and rows at or after b follow every start)
            const uint32_t i0 = c + 4 * lane;
            const uint4 x = vc;
            const uint64_t lsum = (uint64_t)x.x + x.y + x.z + x.w;
            const uint64_t lexcl = warp_incl_scan(lsum) - lsum;
            const uint32_t cexcl = warp_incl_scan(nf) - nf;
            if (f) {
                const uint64_t base = PS1[c >> kChunkLog] + lexcl;
                const uint32_t e[4] = {x.x, x.y, x.z, x.w};
                uint64_t run = 0;
                uint32_t k = off + cexcl;
#pragma unroll
                for (int r = 0; r < 4; r++) {
                    if ((f >> r) & 1u) {
                        vpos[k] = i0 + r;
                        Ps[k] = base + run;
                        k++;
                    }
                    run += e[r];
                }
            }
            off += __shfl_sync(0xffffffffu, cexcl + nf, 31);
        }
    }
}

__global__ void dense_goffv_kernel(const uint32_t *segoff, const uint32_t *dsegf, uint32_t Gd, uint32_t NS,
                                   uint32_t D, uint32_t *goffv) {
    const uint32_t j = blockIdx.x * blockDim.x + threadIdx.x;
    if (j <= Gd) goffv[j] = dsegf[j] < NS ? segoff[dsegf[j]] : D;
}

__global__ void fill_kernel_u32(uint32_t *p, uint32_t n, uint32_t v) {
    const uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i < n) p[i] = v;
}

__global__ void dense_flags_kernel(const uint8_t *vflag, const uint32_t *vpos, uint64_t D, uint32_t *flags) {
    const uint64_t u = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (u < D && vflag[u]) atomicOr(&flags[vpos[u] >> 5], 1u << (vpos[u] & 31));
}

// Selects the dense groups (main stream, one small round trip) and queues the
// count of their distinct values on c.vside; the rest follows from pump().
int DensePath::start(uint64_t n, uint32_t K, double eps, double z, double k2, int clamp) {
    on = false;
    n_ = n;
    phase = 0;
    eps_ = eps;
    z_ = z;
    k2_ = k2;
    clamp_ = clamp;
    if (!value_rows() || K == 0) return STEM_OK;
    cudaStream_t st = c.stream;
    CKS(c.ensure(c.dn_sel, c.cap_dn_sel, (uint64_t)K + 16 * 8));
    uint8_t *sel = (uint8_t *)c.dn_sel;
    unsigned long long *acc = (unsigned long long *)(sel + (((uint64_t)K + 15) & ~15ull));
    CK(cudaMemsetAsync(acc, 0, 16, st));
    dense_select_kernel<<<(unsigned)((K + 7) / 8), 256, 0, st>>>(c.goff, c.t_sorted, K, c.fixed_kernel, value_rows(),
                                                                 value_ratio(), sel, acc);
    c.launches++;
    unsigned long long h[2];
    CK(cudaMemcpyAsync(h, acc, sizeof(h), cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
    if (h[0] == 0) return STEM_OK;
    Gd = (uint32_t)h[0];
    NS = (uint32_t)h[1];
    CKS(c.ensure(c.dn_meta, c.cap_dn_meta, sizeof(uint32_t) * (3 * (Gd + 2) + 2 * (NS + 2)) + 64 +
                                           (scan_tiles((uint64_t)K + NS + 2) + 2) * sizeof(uint64_t)));
    dgrp = (uint32_t *)c.dn_meta;
    dsegf = dgrp + (Gd + 2);
    goffv = dsegf + (Gd + 2);
    segcnt = goffv + (Gd + 2);
    segoff = segcnt + (NS + 2);
    uint64_t *scr = (uint64_t *)(((uintptr_t)(segoff + NS + 2) + 63) & ~(uintptr_t)63);
    if (!c.vside) {
        CK(cudaStreamCreateWithFlags(&c.vside, cudaStreamNonBlocking));
        CK(cudaEventCreateWithFlags(&c.ev_vfork, cudaEventDisableTiming));
        CK(cudaEventCreateWithFlags(&c.ev_vjoin, cudaEventDisableTiming));
        CK(cudaEventCreateWithFlags(&c.ev_vcount, cudaEventDisableTiming));
        CK(cudaMallocHost((void **)&c.h_vcount, sizeof(uint64_t) * 2));
    }
    // STEMROOT_VALUE_SYNC=1: the whole value path on the main stream, before the row levels (a timed stage)
    sync_mode = getenv("STEMROOT_VALUE_SYNC") && getenv("STEMROOT_VALUE_SYNC")[0] == '1';
    vs_ = sync_mode ? st : c.vside;
    cudaStream_t vs = vs_;
    const int tk = sync_mode ? c.stage_begin("root_value") : -1;
    if (!sync_mode) {
        CK(cudaEventRecord(c.ev_vfork, st));
        CK(cudaStreamWaitEvent(vs, c.ev_vfork, 0));
    }
    unsigned long long *tot = acc + 2;
    const uint32_t *goff = c.goff;
    uint32_t *dg = dgrp, *ds = dsegf;
    exclusive_scan<uint64_t>(
        [sel, goff] __device__(uint64_t g) -> uint64_t {
            return sel[g] == 2 ? ((1ull << 32) | ((goff[g + 1] - goff[g] + (goff[g] & 31u) + kWinRows - 1) / kWinRows))
                               : 0ull;
        },
        [dg, ds] __device__(uint64_t g, uint64_t pre, uint64_t v) {
            if (v) {
                dg[pre >> 32] = (uint32_t)g;
                ds[pre >> 32] = (uint32_t)pre;
            }
        },
        K, scr, (uint64_t *)tot, vs, &c.launches);
    const uint32_t ns = NS;
    uint32_t *dsend = dsegf + Gd;
    fill_kernel_u32<<<1, 32, 0, vs>>>(dsend, 1, ns);
    const DenseWin dw{dgrp, dsegf, goff, Gd};
    grid = (unsigned)min((uint64_t)(NS + 7) / 8, (uint64_t)c.sms * 8);
    dense_count_kernel<<<grid, 256, 0, vs>>>(dw, c.t_sorted, NS, segcnt);
    uint32_t *sc = segcnt, *so = segoff;
    exclusive_scan<uint64_t>([sc] __device__(uint64_t s) -> uint64_t { return sc[s]; },
                             [so] __device__(uint64_t s, uint64_t pre, uint64_t) { so[s] = (uint32_t)pre; },
                             NS, scr, (uint64_t *)tot, vs, &c.launches);
    CK(cudaMemcpyAsync(c.h_vcount, tot, sizeof(uint64_t), cudaMemcpyDeviceToHost, vs));
    CK(cudaEventRecord(c.ev_vcount, vs));
    c.launches += 2;
    CK(cudaGetLastError());
    sel_ = sel;
    on = true;
    phase = 1;
    if (sync_mode) {
        CK(cudaEventSynchronize(c.ev_vcount));
        CKS(build());
        uint64_t act = 0;
        CKS(run.finish(&act));
        act_ = act;
        c.stage_end(tk, 12 * act);
    }
    return STEM_OK;
}

// phase 1 -> 2: the distinct count is known: buffers, the value list, the first frontier
int DensePath::build() {
    const uint64_t D = *c.h_vcount;
    D_ = D;
    // growing a buffer frees the old one (an implicit device synchronisation): rare, sizes persist per ctx
    CKS(c.ensure(c.dn_val, c.cap_dn_val, (sizeof(uint32_t) + sizeof(uint64_t) + 1) * (D + 4) + 64));
    vpos = (uint32_t *)c.dn_val;
    uint64_t *Ps = (uint64_t *)(((uintptr_t)(vpos + D + 4) + 15) & ~(uintptr_t)15);
    vflag = (uint8_t *)(Ps + D + 4);
    CKS(c.ensure(c.vr_work, c.cap_vr_work, vr_work_bytes(D)));
    cudaStream_t vs = vs_;
    dense_goffv_kernel<<<(Gd + 256) / 256, 256, 0, vs>>>(segoff, dsegf, Gd, NS, (uint32_t)D, goffv);
    const DenseWin dw{dgrp, dsegf, c.goff, Gd};
    dense_write_kernel<<<grid, 256, 0, vs>>>(dw, c.t_sorted, c.PS1, NS, segoff, vpos, Ps);
    c.launches += 2;
    CK(cudaGetLastError());
    VrSource src{};
    src.kc = vpos;
    src.Ps = Ps;
    src.goffv = goffv;
    src.dgrp = dgrp;
    src.goff = c.goff;
    src.G = Gd;
    CKS(run.setup(src, D, eps_, z_, k2_, clamp_, vflag, vs));
    phase = 2;
    return STEM_OK;
}

int DensePath::pump() {
    if (!on || sync_mode) return STEM_OK;
    if (phase == 1) {
        const cudaError_t q = cudaEventQuery(c.ev_vcount);
        if (q == cudaErrorNotReady) {
            (void)cudaGetLastError();
            return STEM_OK;
        }
        CK(q);
        CKS(build());
    }
    return run.pump(false);
}

// Completes the value tree, sets its leaf starts in the row flags and joins the streams.
int DensePath::finish(uint32_t *flags) {
    if (!on) return STEM_OK;
    if (phase == 1) {
        CK(cudaEventSynchronize(c.ev_vcount));
        CKS(build());
    }
    uint64_t act = act_;
    if (!sync_mode) CKS(run.finish(&act));
    cudaStream_t vs = vs_;
    if (D_) dense_flags_kernel<<<(unsigned)((D_ + 255) / 256), 256, 0, vs>>>(vflag, vpos, D_, flags);
    c.launches += 1 + run.launches;
    if (!sync_mode) {
        CK(cudaEventRecord(c.ev_vjoin, vs));
        CK(cudaStreamWaitEvent(c.stream, c.ev_vjoin, 0));
    }
    CK(cudaGetLastError());
    c.stats.active_rows += act;
    c.stats.value_groups += Gd;
    c.stats.value_count += D_;
    if (run.levels > c.stats.value_levels) c.stats.value_levels = run.levels;
    on = false;
    return STEM_OK;
}

}  // namespace sr
