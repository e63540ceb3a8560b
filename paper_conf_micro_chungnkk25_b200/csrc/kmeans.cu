// kmeans.cu -- ROOT with k-ary splits, split = 3 (R29): each
// frontier cluster is divided by the exact optimal 1-D k-means ("a
// clustering method (e.g., k-means) ... any number above 2 works well") into
// min(k, #distinct values) groups of consecutive distinct values, and the
// split is kept iff Eq. 8 over the groups beats Eq. 7.
//
// The k-means is the dynamic program over the cluster's distinct values
//   F[1][b] = S(0,b)^2 / n(0,b),  F[j][b] = max_a F[j-1][a] + S(a,b)^2 / n(a,b)
// (maximising sum_g S_g^2 / n_g = minimising the SSE), evaluated in fp64 in its
// between-group form (km_between below) and only for b = d in the last layer.  The group cost obeys
// the quadrangle inequality, so the smallest optimal a is non-decreasing in b
// and each layer is solved by divide and conquer in O(d log d): one warp per
// cluster, 32 candidate a per step.  Values are fp64; candidates within 2^-40
// of the best are compared EXACTLY (the prefix partitions rebuilt from the
// argmax table, sums of fractions in 768-bit integers), and ties keep the
// smaller a -- the oracle's rule (smallest last cut, then the one before).
//
// Distinct values: row i starts one when it starts a kernel group or
// t[i-1] < t[i]; their positions and exact prefix sums are built once per
// plan for the whole trace, so a cluster's distinct values are the contiguous
// slice of that list between its bounds (a cut never separates equal times).
#include "internal.h"

namespace sr {

constexpr int kKmMax = 8;              // largest kmeans_k
constexpr int kKmLimbs = 12;           // 768-bit integers (sums of <= 8 fractions, cross-multiplied)

// ---------------------------------------------------------------- exact fractions (rare near-tie path)
struct KBig { uint64_t w[kKmLimbs]; };

__device__ __noinline__ void kbig_mul(const KBig &a, const KBig &b, KBig &r) {
    uint64_t o[kKmLimbs];
    for (int i = 0; i < kKmLimbs; i++) o[i] = 0;
    for (int i = 0; i < kKmLimbs; i++) {
        if (!a.w[i]) continue;
        uint64_t carry = 0;
        for (int j = 0; i + j < kKmLimbs; j++) {
            const uint64_t lo = a.w[i] * b.w[j], hi = __umul64hi(a.w[i], b.w[j]);
            uint64_t s = o[i + j] + lo;
            uint64_t c1 = s < lo;
            s += carry;
            c1 += s < carry;
            o[i + j] = s;
            carry = hi + c1;
        }
    }
    for (int i = 0; i < kKmLimbs; i++) r.w[i] = o[i];
}

__device__ __forceinline__ void kbig_add(KBig &a, const KBig &b) {
    uint64_t carry = 0;
    for (int i = 0; i < kKmLimbs; i++) {
        uint64_t s = a.w[i] + b.w[i];
        const uint64_t c1 = s < a.w[i];
        s += carry;
        carry = c1 + (s < carry);
        a.w[i] = s;
    }
}

__device__ __forceinline__ int kbig_cmp(const KBig &a, const KBig &b) {
    for (int i = kKmLimbs - 1; i >= 0; i--)
        if (a.w[i] != b.w[i]) return a.w[i] < b.w[i] ? -1 : 1;
    return 0;
}

struct KFrac { KBig num, den; };

// f + S^2 / n
__device__ __noinline__ void kfrac_add(KFrac &f, uint64_t S, uint64_t n) {
    KBig bn{}, s2{}, a, b;
    bn.w[0] = n;
    s2.w[0] = S * S;
    s2.w[1] = __umul64hi(S, S);
    kbig_mul(f.num, bn, a);
    kbig_mul(s2, f.den, b);
    kbig_add(a, b);
    f.num = a;
    kbig_mul(f.den, bn, b);
    f.den = b;
}

__device__ __noinline__ int kfrac_cmp(const KFrac &x, const KFrac &y) {
    KBig l, r;
    kbig_mul(x.num, y.den, l);
    kbig_mul(y.num, x.den, r);
    return kbig_cmp(l, r);
}

struct KmArgs {
    const uint32_t *f_lo, *f_hi;
    const uint64_t *ctot;          // packed (count << 32 | rows) of the frontier
    const uint32_t *dpos;          // [D + 1] rows starting a distinct value (dpos[D] = n)
    const uint64_t *dP;            // [D + 1] exact sum of t before them
    uint64_t D;
    double *F;                     // [k + 1][D + 1] fp64 DP values (layers 1..k): the high part of
    double *Flo;                   // [k + 1][D + 1] their double-double low part
    uint32_t *arg;                 // [k + 1][D + 1] argmax (distinct index relative to the cluster)
    uint32_t k;
    uint32_t *cutk;                // [cluster][kKmMax - 1] cuts relative to lo
    uint32_t *ngrp;                // [cluster] groups (0: leaf)
};

struct KmCluster {
    uint64_t D0, lo;
    uint32_t d;
};

__device__ __forceinline__ uint64_t km_pos(const KmArgs &a, const KmCluster &c, uint32_t u) {
    return (uint64_t)a.dpos[c.D0 + u] - c.lo;
}
__device__ __forceinline__ uint64_t km_P(const KmArgs &a, const KmCluster &c, uint32_t u) {
    return a.dP[c.D0 + u] - a.dP[c.D0];
}

// exact value of F[j-1][a] + S(a,b)^2/n(a,b): the prefix partition of the first
// a distinct values into j - 1 groups rebuilt from the argmax table
__device__ __noinline__ void km_exact(const KmArgs &g, const KmCluster &c, uint32_t j, uint32_t a, uint32_t b,
                                      KFrac &out) {
    for (int i = 0; i < kKmLimbs; i++) out.num.w[i] = out.den.w[i] = 0;
    out.den.w[0] = 1;
    const size_t L = g.D + 1;
    uint32_t hi = a;
    for (uint32_t l = j - 1; l >= 1; l--) {
        const uint32_t lo = l == 1 ? 0u : g.arg[(size_t)l * L + c.D0 + hi];
        kfrac_add(out, km_P(g, c, hi) - km_P(g, c, lo), km_pos(g, c, hi) - km_pos(g, c, lo));
        hi = lo;
        if (l == 1) break;
    }
    kfrac_add(out, km_P(g, c, b) - km_P(g, c, a), km_pos(g, c, b) - km_pos(g, c, a));
}

// ---------------------------------------------------------------- the DP, level-synchronous divide and conquer
// Layer j of every active cluster at once: a subproblem (cluster, b range,
// a range) takes b = mid of its range, finds the best a for it and hands the
// two halves (with the narrowed a ranges) to the next round.  One round per
// recursion depth for all clusters together (about log2 of the largest d);
// long a ranges get a block, short ones a warp.
struct KmSub {
    uint32_t c, blo, bhi, alo, ahi, pad;
};

struct KmMeta {          // per frontier cluster
    uint64_t D0, lo;
    uint32_t d, K;
};

// Between-group form of the DP (the fp64 filter's values): G[j][b] = F[j][b] -
// S(0,b)^2/n(0,b) = max_a G[j-1][a] + T(a,b), G[1][b] = 0, with
// T(a,b) = S(0,a)^2/n(0,a) + S(a,b)^2/n(a,b) - S(0,b)^2/n(0,b)
//        = (n(a,b) S(0,a) - n(0,a) S(a,b))^2 / (n(0,a) n(a,b) n(0,b)),
// the numerator exact in 128 bits (<= 0 inside the difference for sorted
// values).  For a fixed b the order of G[j-1][a] + T(a,b) is the order of
// F[j-1][a] + S(a,b)^2/n(a,b) (they differ by a constant), so the exact
// comparison of near ties is unchanged; but G has no large common part, so
// the 2^-40 filter flags far fewer near ties than F = sum S^2/n did (C5: the
// sums are ~1e20 while candidates differ by ~1e9).
__device__ __forceinline__ double km_between(const KmArgs &g, const KmCluster &c, uint32_t a, uint32_t b) {
    const uint64_t na = km_pos(g, c, a), nb = km_pos(g, c, b), nab = nb - na;
    const uint64_t Sa = km_P(g, c, a), Sab = km_P(g, c, b) - Sa;
    const u128 l = (u128)na * Sab, r = (u128)nab * Sa;   // n(0,a) S(a,b) >= n(a,b) S(0,a) for sorted values
    const u128 D = l >= r ? l - r : r - l;
    const double dD = rn128(D);
    return __ddiv_rn(__dmul_rn(dD, dD), __dmul_rn(__dmul_rn(rn64(na), rn64(nab)), rn64(nb)));
}

__device__ __noinline__ uint32_t km_exact_best(const KmArgs &g, const KmCluster &c, uint32_t j, uint32_t b,
                                               const uint32_t *list, uint32_t m);

// ---- double-double (~2^-100 relative) values: the second filter between the
// fp64 scan (2^-40 band) and the exact 768-bit comparison
struct KDD {
    double hi, lo;
};
__device__ __forceinline__ KDD kdd_qsum(double a, double b) {
    const double s = __dadd_rn(a, b);
    return KDD{s, __dsub_rn(b, __dsub_rn(s, a))};
}
__device__ __forceinline__ KDD kdd_sum(double a, double b) {
    const double s = __dadd_rn(a, b), bb = __dsub_rn(s, a);
    return KDD{s, __dadd_rn(__dsub_rn(a, __dsub_rn(s, bb)), __dsub_rn(b, bb))};
}
__device__ __forceinline__ KDD kdd_add(KDD a, KDD b) {
    KDD s = kdd_sum(a.hi, b.hi);
    const KDD t = kdd_sum(a.lo, b.lo);
    s = kdd_qsum(s.hi, __dadd_rn(s.lo, t.hi));
    return kdd_qsum(s.hi, __dadd_rn(s.lo, t.lo));
}
__device__ __forceinline__ KDD kdd_mul(KDD a, KDD b) {
    const double p = __dmul_rn(a.hi, b.hi);
    double e = __fma_rn(a.hi, b.hi, -p);
    e = __dadd_rn(e, __dadd_rn(__dmul_rn(a.hi, b.lo), __dmul_rn(a.lo, b.hi)));
    return kdd_qsum(p, e);
}
__device__ __forceinline__ KDD kdd_mul_d(KDD a, double b) {
    const double p = __dmul_rn(a.hi, b);
    const double e = __dadd_rn(__fma_rn(a.hi, b, -p), __dmul_rn(a.lo, b));
    return kdd_qsum(p, e);
}
__device__ __forceinline__ KDD kdd_div(KDD a, KDD b) {
    const double q1 = __ddiv_rn(a.hi, b.hi);
    KDD r = kdd_add(a, kdd_mul_d(b, -q1));
    const double q2 = __ddiv_rn(r.hi, b.hi);
    r = kdd_add(r, kdd_mul_d(b, -q2));
    const double q3 = __ddiv_rn(r.hi, b.hi);
    return kdd_add(kdd_qsum(q1, q2), KDD{q3, 0.0});
}
__device__ __forceinline__ KDD kdd_u128(u128 x) {   // exact for x < 2^106
    const uint64_t h = (uint64_t)(x >> 53), l = (uint64_t)x & ((1ull << 53) - 1);
    return kdd_sum(__dmul_rn((double)h, 0x1p53), (double)l);
}
__device__ __forceinline__ bool kdd_gt(KDD a, KDD b) { return a.hi > b.hi || (a.hi == b.hi && a.lo > b.lo); }

// G[j-1][a] + T(a,b) in double-double
__device__ __forceinline__ KDD km_value_dd(const KmArgs &g, const KmCluster &c, uint32_t j, uint32_t a, uint32_t b) {
    const uint64_t na = km_pos(g, c, a), nb = km_pos(g, c, b), nab = nb - na;
    const uint64_t Sa = km_P(g, c, a), Sab = km_P(g, c, b) - Sa;
    const u128 l = (u128)na * Sab, r = (u128)nab * Sa;
    const KDD D = kdd_u128(l >= r ? l - r : r - l);   // < 2^96
    const KDD T = kdd_div(kdd_mul(D, D), kdd_u128((u128)(na * nab) * nb));
    const size_t idx = (size_t)(j - 1) * (g.D + 1) + c.D0 + a;
    return kdd_add(KDD{g.F[idx], g.Flo[idx]}, T);
}

// The winner among near-tie candidates (ascending): by double-double values
// when one beats every other by more than 2^-90 relative (their errors are
// below 2^-96), else by the exact comparison
__device__ __noinline__ uint32_t km_near_best(const KmArgs &g, const KmCluster &c, uint32_t j, uint32_t b,
                                              const uint32_t *list, uint32_t m) {
    if (m == 1) return list[0];
    KDD v1 = km_value_dd(g, c, j, list[0], b), v2{-1.0, 0.0};
    uint32_t a1 = list[0];
    for (uint32_t i = 1; i < m; i++) {
        const KDD v = km_value_dd(g, c, j, list[i], b);
        if (kdd_gt(v, v1)) { v2 = v1; v1 = v; a1 = list[i]; }
        else if (kdd_gt(v, v2)) v2 = v;
    }
    const KDD thr = kdd_add(v1, KDD{__dmul_rn(-v1.hi, 0x1p-90), 0.0});
    if (kdd_gt(thr, v2)) return a1;
    return km_exact_best(g, c, j, b, list, m);
}

__device__ __forceinline__ double km_value(const KmArgs &g, const KmCluster &c, uint32_t j, uint32_t a, uint32_t b) {
    return __dadd_rn(g.F[(size_t)(j - 1) * (g.D + 1) + c.D0 + a], km_between(g, c, a, b));
}

// exact winner among the candidates a in list[0..m) (ascending), any thread
__device__ __noinline__ uint32_t km_exact_best(const KmArgs &g, const KmCluster &c, uint32_t j, uint32_t b,
                                               const uint32_t *list, uint32_t m) {
    KFrac bf, cf;
    uint32_t best = list[0];
    km_exact(g, c, j, best, b, bf);
    for (uint32_t i = 1; i < m; i++) {
        km_exact(g, c, j, list[i], b, cf);
        if (kfrac_cmp(cf, bf) > 0) {
            bf = cf;
            best = list[i];
        }
    }
    return best;
}

// Subproblems travel in two lists by the length of their a range (short: a
// warp each, long: a block each), so neither kernel walks the other's entries.
struct KmStep {
    KmArgs g;
    const KmMeta *meta;
    const KmSub *cur[2];      // [short, long]
    const uint32_t *ncur[2];
    KmSub *nxt[2];
    uint32_t *nnxt[2];
    uint32_t j;
};

constexpr uint32_t kKmLong = 512;   // a ranges longer than this get a block
#ifndef SR_KM_LEAFA
#define SR_KM_LEAFA 64
#endif
constexpr uint32_t kKmLeafA = SR_KM_LEAFA;   // subproblems of <= 32 b and < this many a: solved whole by one warp
constexpr int kKmNear = 256;        // near-tie candidates resolved exactly per subproblem

// the list a subproblem belongs to: 1 (long) when its b = mid scans more than kKmLong candidates
__device__ __forceinline__ int km_cls(const KmSub &x) {
    const uint32_t mid = x.blo + (x.bhi - x.blo) / 2;
    return min(x.ahi, mid - 1) - x.alo + 1 > kKmLong ? 1 : 0;
}
__device__ __forceinline__ void km_push(KmSub *const *lst, uint32_t *const *cnt, const KmSub &x) {
    const int k = km_cls(x);
    lst[k][atomicAdd(cnt[k], 1u)] = x;
}

__device__ __forceinline__ void km_emit(const KmStep &s, const KmSub &x, uint32_t mid, uint32_t a) {
    if (mid > x.blo) km_push(s.nxt, s.nnxt, KmSub{x.c, x.blo, mid - 1, x.alo, a, 0});
    if (mid < x.bhi) km_push(s.nxt, s.nnxt, KmSub{x.c, mid + 1, x.bhi, a, x.ahi, 0});
}

__device__ __forceinline__ KmCluster km_cluster(const KmMeta &m) {
    KmCluster c;
    c.D0 = m.D0;
    c.lo = m.lo;
    c.d = m.d;
    return c;
}

// running (best value, its smallest a, second best value) of a candidate scan;
// the second best counts an equal best value, so a unique winner is certain
// when second < best (1 - 2^-40) and the near-tie pass can be skipped
struct KmTop {
    double v1, v2;
    uint32_t a1;
};
__device__ __forceinline__ void km_top_add(KmTop &t, double v, uint32_t a) {
    if (v > t.v1) { t.v2 = t.v1; t.v1 = v; t.a1 = a; }
    else if (v == t.v1) { t.v2 = v; if (a < t.a1) t.a1 = a; }
    else if (v > t.v2) t.v2 = v;
}
__device__ __forceinline__ KmTop km_top_merge(const KmTop &x, const KmTop &y) {
    KmTop r;
    if (x.v1 > y.v1) { r.v1 = x.v1; r.a1 = x.a1; r.v2 = fmax(x.v2, y.v1); }
    else if (y.v1 > x.v1) { r.v1 = y.v1; r.a1 = y.a1; r.v2 = fmax(y.v2, x.v1); }
    else { r.v1 = x.v1; r.a1 = min(x.a1, y.a1); r.v2 = x.v1; }
    return r;
}
__device__ __forceinline__ KmTop km_top_warp(KmTop t) {
#pragma unroll
    for (int o = 16; o; o >>= 1) {
        KmTop y;
        y.v1 = __shfl_xor_sync(0xffffffffu, t.v1, o);
        y.v2 = __shfl_xor_sync(0xffffffffu, t.v2, o);
        y.a1 = __shfl_xor_sync(0xffffffffu, t.a1, o);
        t = km_top_merge(t, y);
    }
    return t;
}

// subproblems with long a ranges: one block each
__global__ void __launch_bounds__(256) km_step_block_kernel(KmStep s) {
    __shared__ double s_v[8], s_v2[8];
    __shared__ uint32_t s_a[8];
    __shared__ uint32_t s_list[kKmNear];
    __shared__ uint32_t s_m;
    const uint32_t n = *s.ncur[1];
    const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
    for (uint32_t i = blockIdx.x; i < n; i += gridDim.x) {
        const KmSub x = s.cur[1][i];
        const uint32_t mid = x.blo + (x.bhi - x.blo) / 2;
        const uint32_t a0 = x.alo, a1 = min(x.ahi, mid - 1);
        const KmCluster c = km_cluster(s.meta[x.c]);
        KmTop tp{-1.0, -1.0, 0xFFFFFFFFu};
        for (uint32_t a = a0 + tid; a <= a1; a += 256) km_top_add(tp, km_value(s.g, c, s.j, a, mid), a);
        tp = km_top_warp(tp);
        if (lane == 0) { s_v[w] = tp.v1; s_v2[w] = tp.v2; s_a[w] = tp.a1; }
        if (tid == 0) s_m = 0;
        __syncthreads();
        KmTop top{s_v[0], s_v2[0], s_a[0]};
        for (int k = 1; k < 8; k++) top = km_top_merge(top, KmTop{s_v[k], s_v2[k], s_a[k]});
        const double thr = __dmul_rn(top.v1, 1.0 - 0x1p-40);
        const bool unique = top.v2 < thr;   // every other candidate is below the near-tie band
        if (!unique)
            for (uint32_t a = a0 + tid; a <= a1; a += 256)
                if (km_value(s.g, c, s.j, a, mid) >= thr) {
                    const uint32_t q = atomicAdd(&s_m, 1u);
                    if (q < (uint32_t)kKmNear) s_list[q] = a;
                }
        __syncthreads();
        if (tid == 0) {
            if (unique) { s_list[0] = top.a1; s_m = 1; }
            uint32_t m = min(s_m, (uint32_t)kKmNear), best;
            for (uint32_t p = 1; p < m; p++)   // ascending a (insertion sort of a few entries)
                for (uint32_t q = p; q > 0 && s_list[q - 1] > s_list[q]; q--) {
                    const uint32_t t = s_list[q]; s_list[q] = s_list[q - 1]; s_list[q - 1] = t;
                }
            best = km_near_best(s.g, c, s.j, mid, s_list, m);
            const size_t L = s.g.D + 1;
            const KDD vb = km_value_dd(s.g, c, s.j, best, mid);
            s.g.F[(size_t)s.j * L + c.D0 + mid] = vb.hi;
            s.g.Flo[(size_t)s.j * L + c.D0 + mid] = vb.lo;
            s.g.arg[(size_t)s.j * L + c.D0 + mid] = best;
            km_emit(s, x, mid, best);
            if (s_m > (uint32_t)kKmNear) atomicOr(s.g.ngrp + x.c, 0x80000000u);   // flagged: too many near ties
        }
        __syncthreads();
    }
}

// subproblems with short a ranges: one warp each
__global__ void __launch_bounds__(256) km_step_warp_kernel(KmStep s) {
    __shared__ uint32_t s_list[8][kKmNear];   // 8 KB
    const uint32_t n = *s.ncur[0];
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    const uint64_t nwarps = ((uint64_t)gridDim.x * blockDim.x) >> 5;
    for (uint64_t i = ((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; i < n; i += nwarps) {
        const KmSub x = s.cur[0][i];
        const KmCluster c = km_cluster(s.meta[x.c]);
        if (x.bhi - x.blo < 32 && x.ahi - x.alo < kKmLeafA && !x.pad) {
            // the whole sub-tree at once: lane i solves b = blo + i over the
            // subproblem's a range (it holds every b's smallest optimal a), one
            // scan per lane; a lane whose best is not unique by 2^-40 goes back
            // to the list as a single-b subproblem (near-tie path next round)
            const uint32_t b = x.blo + lane;
            if (b <= x.bhi) {
                KmTop tp{-1.0, -1.0, 0xFFFFFFFFu};
                const uint32_t ae = min(x.ahi, b - 1);
                for (uint32_t a = x.alo; a <= ae; a++) km_top_add(tp, km_value(s.g, c, s.j, a, b), a);
                if (tp.v2 < __dmul_rn(tp.v1, 1.0 - 0x1p-40)) {
                    const size_t L = s.g.D + 1, idx = (size_t)s.j * L + c.D0 + b;
                    const KDD vb = km_value_dd(s.g, c, s.j, tp.a1, b);
                    s.g.F[idx] = vb.hi;
                    s.g.Flo[idx] = vb.lo;
                    s.g.arg[idx] = tp.a1;
                } else {
                    km_push(s.nxt, s.nnxt, KmSub{x.c, b, b, x.alo, x.ahi, 1});   // pad = 1: never a leaf again
                }
            }
            continue;
        }
        const uint32_t mid = x.blo + (x.bhi - x.blo) / 2;
        const uint32_t a0 = x.alo, a1 = min(x.ahi, mid - 1);
        KmTop tp{-1.0, -1.0, 0xFFFFFFFFu};
        for (uint32_t a = a0 + lane; a <= a1; a += 32) km_top_add(tp, km_value(s.g, c, s.j, a, mid), a);
        tp = km_top_warp(tp);
        const double thr = __dmul_rn(tp.v1, 1.0 - 0x1p-40);
        uint32_t m = 0;
        if (tp.v2 < thr) {   // a unique winner: no near-tie pass
            if (lane == 0) s_list[w][0] = tp.a1;
            m = 1;
        } else
        for (uint32_t base = a0; base <= a1; base += 32) {   // near-tie candidates, ascending
            const uint32_t a = base + lane;
            const bool near = a <= a1 && km_value(s.g, c, s.j, a, mid) >= thr;
            const uint32_t bm = __ballot_sync(0xffffffffu, near);
            if (near) {
                const uint32_t q = m + __popc(bm & ((1u << lane) - 1));
                if (q < (uint32_t)kKmNear) s_list[w][q] = a;
            }
            m += __popc(bm);
        }
        __syncwarp();
        if (lane == 0) {
            const uint32_t mm = min(m, (uint32_t)kKmNear);
            const uint32_t best = km_near_best(s.g, c, s.j, mid, s_list[w], mm);
            const size_t L = s.g.D + 1;
            const KDD vb = km_value_dd(s.g, c, s.j, best, mid);
            s.g.F[(size_t)s.j * L + c.D0 + mid] = vb.hi;
            s.g.Flo[(size_t)s.j * L + c.D0 + mid] = vb.lo;
            s.g.arg[(size_t)s.j * L + c.D0 + mid] = best;
            km_emit(s, x, mid, best);
            if (m > (uint32_t)kKmNear) atomicOr(s.g.ngrp + x.c, 0x80000000u);
        }
        __syncwarp();
    }
}

// per cluster: its distinct-value slice, K = min(k, d), layer 1, and the
// layer-2 subproblem; one warp per cluster
struct KmLists {
    KmSub *lst[2];
    uint32_t *cnt[2];
};
__global__ void __launch_bounds__(256) km_prep_kernel(KmArgs g, KmMeta *meta, KmLists L) {
    const uint32_t C = (uint32_t)(*g.ctot >> 32);
    const int lane = threadIdx.x & 31;
    const uint64_t nwarps = ((uint64_t)gridDim.x * blockDim.x) >> 5;
    for (uint64_t ci = ((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; ci < C; ci += nwarps) {
        const uint64_t lo = g.f_lo[ci], hi = g.f_hi[ci];
        KmMeta m;
        m.lo = lo;
        m.D0 = lower_bound(g.dpos, g.D + 1, (uint32_t)lo);
        m.d = (uint32_t)(lower_bound(g.dpos, g.D + 1, (uint32_t)hi) - m.D0);
        m.K = min(g.k, m.d);
        const KmCluster c = km_cluster(m);
        for (uint32_t b = 1 + lane; b <= m.d; b += 32) {   // G[1][b] = 0 (one group)
            g.F[(g.D + 1) + c.D0 + b] = 0.0;
            g.Flo[(g.D + 1) + c.D0 + b] = 0.0;
        }
        if (lane == 0) {
            meta[ci] = m;
            g.ngrp[ci] = 0;
            // the last layer needs b = d only (the backtrack starts there)
            if (m.K >= 2) km_push(L.lst, L.cnt, KmSub{(uint32_t)ci, m.K == 2 ? m.d : 2, m.d, 1, m.d - 1, 0});
        }
    }
}

// the next layer's root subproblems
__global__ void km_layer_kernel(const uint64_t *ctot, const KmMeta *meta, uint32_t j, KmLists L) {
    const uint64_t ci = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (ci >= (*ctot >> 32)) return;
    const KmMeta m = meta[ci];
    if (m.K >= j) km_push(L.lst, L.cnt, KmSub{(uint32_t)ci, m.K == j ? m.d : j, m.d, j - 1, m.d - 1, 0});
}

// backtrack the cuts
__global__ void km_finish_kernel(KmArgs g, const KmMeta *meta) {
    const uint64_t ci = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (ci >= (*g.ctot >> 32)) return;
    const KmMeta m = meta[ci];
    if (g.ngrp[ci] & 0x80000000u) return;   // too many near ties for the exact list: reported as an error
    if (m.K < 2) { g.ngrp[ci] = 0; return; }
    const KmCluster c = km_cluster(m);
    const size_t L = g.D + 1;
    uint32_t b = m.d;
    for (uint32_t j = m.K; j >= 2; j--) {
        b = g.arg[(size_t)j * L + c.D0 + b];
        g.cutk[ci * (kKmMax - 1) + (j - 2)] = (uint32_t)km_pos(g, c, b);
    }
    g.ngrp[ci] = m.K;
}

// ---------------------------------------------------------------- decision and children (Eq. 7 vs Eq. 8)
struct KdArgs {
    const uint32_t *f_lo, *f_hi;
    const uint64_t *f_S;
    const u128 *f_Q;
    const uint64_t *ctot;
    const uint32_t *cutk, *ngrp;
    const uint64_t *PS1;
    const u128 *PS2;
    const uint32_t *t;
    uint32_t *flags;
    uint32_t *nlo, *nhi;
    uint64_t *nS;
    u128 *nQ;
    uint64_t *total;
    double eps, z, k2;
    int clamp;
    uint32_t *err;
};

__device__ __forceinline__ double km_eq6(double g, double mu, double V, int clamp) {
    if (V == 0.0) return clamp ? 1.0 : 0.0;
    double m = ceil(__dmul_rn(g, __dsqrt_rn(__ddiv_rn(V, mu))));
    if (clamp && m < 1.0) m = 1.0;
    return m;
}

__global__ void __launch_bounds__(128) kmeans_decide_kernel(KdArgs a) {
    const uint64_t c = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (c >= (*a.ctot >> 32)) return;
    const uint32_t G = a.ngrp[c];
    if (G & 0x80000000u) {   // more than kKmNear exact-tie candidates in one DP cell
        atomicOr(a.err, 8u);
        return;
    }
    if (G < 2) return;
    const uint64_t lo = a.f_lo[c], hi = a.f_hi[c], n = hi - lo, S = a.f_S[c];
    const u128 Q = a.f_Q[c];
    // group boundaries and moments
    uint64_t bnd[kKmMax + 1], gS[kKmMax];
    u128 gQ[kKmMax];
    bnd[0] = lo;
    for (uint32_t i = 1; i < G; i++) bnd[i] = lo + a.cutk[c * (kKmMax - 1) + (i - 1)];
    bnd[G] = hi;
    uint64_t s0, sp;
    u128 q0, qp;
    pref12(a.PS1, a.PS2, a.t, lo, s0, q0);
    sp = s0;
    qp = q0;
    for (uint32_t i = 0; i < G; i++) {
        uint64_t s1;
        u128 q1;
        if (i + 1 == G) { s1 = s0 + S; q1 = q0 + Q; }
        else pref12(a.PS1, a.PS2, a.t, bnd[i + 1], s1, q1);
        gS[i] = s1 - sp;
        gQ[i] = q1 - qp;
        sp = s1;
        qp = q1;
    }
    // Eq. 7: tau_old = m * Xbar, m from Eq. 3
    const u128 V = (u128)n * Q - (u128)S * S;
    const double mu = __ddiv_rn(rn64(S), rn64(n));
    double m_old;
    if (V == 0) m_old = a.clamp ? 1.0 : 0.0;
    else {
        const double dS = rn64(S);
        m_old = ceil(__dmul_rn(__ddiv_rn(rn128(V), __dmul_rn(dS, dS)), a.k2));
        if (a.clamp && m_old < 1.0) m_old = 1.0;
    }
    const double tau_old = __dmul_rn(m_old, mu);
    // Eq. 8 over the G children, Eq. 6 with c from the parent's total, left to right
    double gmu[kKmMax], gV[kKmMax];
    for (uint32_t i = 0; i < G; i++) {
        const uint64_t ni = bnd[i + 1] - bnd[i];
        gmu[i] = __ddiv_rn(rn64(gS[i]), rn64(ni));
        gV[i] = rn128((u128)ni * gQ[i] - (u128)gS[i] * gS[i]);
    }
    const double w = __ddiv_rn(__dmul_rn(a.eps, rn64(S)), a.z);
    const double cc = __dmul_rn(w, w);
    double ssum = 0.0;
    for (uint32_t i = 0; i < G; i++) {
        const double term = __dsqrt_rn(__dmul_rn(gmu[i], gV[i]));
        ssum = i == 0 ? term : __dadd_rn(ssum, term);
    }
    const double gg = __ddiv_rn(ssum, cc);
    double tau_new = 0.0;
    for (uint32_t i = 0; i < G; i++) {
        const double term = __dmul_rn(km_eq6(gg, gmu[i], gV[i], a.clamp), gmu[i]);
        tau_new = i == 0 ? term : __dadd_rn(tau_new, term);
    }
    if (!(tau_new < tau_old)) return;   // strict: a leaf
    for (uint32_t i = 0; i < G; i++) {
        if (i > 0) atomicOr(&a.flags[bnd[i] >> 5], 1u << (bnd[i] & 31));
        const uint64_t x0 = bnd[i], x1 = bnd[i + 1];
        if (x1 - x0 >= 2 && a.t[x0] != a.t[x1 - 1]) {
            const uint64_t slot = atomicAdd((unsigned long long *)a.total,
                                            (unsigned long long)((1ull << 32) | (x1 - x0))) >> 32;
            a.nlo[slot] = (uint32_t)x0;
            a.nhi[slot] = (uint32_t)x1;
            a.nS[slot] = gS[i];
            a.nQ[slot] = gQ[i];
        }
    }
}

// ---------------------------------------------------------------- setup kernels
// initial frontier: the non-trivial kernel groups (order immaterial)
__global__ void kmeans_init_kernel(const uint32_t *goff, uint32_t K, const uint32_t *t, const uint64_t *PS1,
                                   const u128 *PS2, uint32_t *nlo, uint32_t *nhi, uint64_t *nS, u128 *nQ,
                                   uint64_t *total) {
    const uint64_t g = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (g >= K) return;
    const uint32_t lo = goff[g], hi = goff[g + 1];
    if (hi - lo < 2 || t[lo] == t[hi - 1]) return;
    uint64_t s0, s1;
    u128 q0, q1;
    pref12(PS1, PS2, t, lo, s0, q0);
    pref12(PS1, PS2, t, hi, s1, q1);
    const uint64_t slot = atomicAdd((unsigned long long *)total, (unsigned long long)((1ull << 32) | (hi - lo))) >> 32;
    nlo[slot] = lo;
    nhi[slot] = hi;
    nS[slot] = s1 - s0;
    nQ[slot] = q1 - q0;
}

__global__ void kmeans_sentinel_kernel(const uint64_t *PS1, const uint32_t *t, uint64_t n, uint32_t *dpos,
                                       uint64_t *dP) {
    if (threadIdx.x == 0) {
        *dpos = (uint32_t)n;
        *dP = pref1(PS1, t, n);
    }
}

int root_levels_kmeans(Ctx &c, uint64_t n, uint32_t K, double eps, double z, double k2, int clamp, uint32_t kk) {
    cudaStream_t st = c.stream;
    if (kk < 2 || kk > (uint32_t)kKmMax) return STEM_E_INVAL;
    CKS(stem_only_leaves(c, n, K));   // group starts in the leaf bitmap
    // distinct-value starts of the whole trace: positions and exact prefix sums
    CKS(c.ensure(c.km_dpos, c.cap_km_dpos, sizeof(uint32_t) * (n + 2)));
    CKS(c.ensure(c.km_dP, c.cap_km_dP, sizeof(uint64_t) * (n + 2)));
    CKS(c.ensure(c.scan_scratch, c.cap_scan, (scan_tiles(n) + 1) * sizeof(uint64_t)));
    {
        const uint32_t *t = c.t_sorted, *fl = c.flags;
        const uint64_t *PS1 = c.PS1;
        uint32_t *dpos = c.km_dpos;
        uint64_t *dP = c.km_dP;
        exclusive_scan<uint64_t>(
            [t, fl] __device__(uint64_t i) -> uint64_t {
                return (i == 0 || ((fl[i >> 5] >> (i & 31)) & 1u) || t[i - 1] < t[i]) ? 1ull : 0ull;
            },
            [t, dpos, dP, PS1] __device__(uint64_t i, uint64_t pre, uint64_t v) {
                if (!v) return;
                dpos[pre] = (uint32_t)i;
                dP[pre] = pref1(PS1, t, i);
            },
            n, (uint64_t *)c.scan_scratch, &c.scalars->scan_total64, st, &c.launches);
    }
    uint64_t D = 0;
    CK(cudaMemcpyAsync(&D, &c.scalars->scan_total64, sizeof(uint64_t), cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
    kmeans_sentinel_kernel<<<1, 32, 0, st>>>(c.PS1, c.t_sorted, n, c.km_dpos + D, c.km_dP + D);   // dpos[D] = n
    c.launches++;
    CKS(c.ensure(c.km_F, c.cap_km_F, 2 * sizeof(double) * (size_t)(kk + 1) * (D + 1)));   // high and low parts
    CKS(c.ensure(c.km_arg, c.cap_km_arg, sizeof(uint32_t) * (size_t)(kk + 1) * (D + 1)));
    // initial frontier
    uint64_t Cmax = (uint64_t)K + 1;
    for (int b = 0; b < 2; b++) {
        CKS(c.ensure(c.f_lo[b], c.cap_flo[b], sizeof(uint32_t) * Cmax));
        CKS(c.ensure(c.f_hi[b], c.cap_fhi[b], sizeof(uint32_t) * Cmax));
        CKS(c.ensure(c.f_S[b], c.cap_fS[b], sizeof(uint64_t) * Cmax));
        CKS(c.ensure(c.f_Q[b], c.cap_fQ[b], sizeof(u128) * Cmax));
    }
    CK(cudaMemsetAsync(&c.scalars->ftot[0], 0, sizeof(uint64_t), st));
    if (K) {
        kmeans_init_kernel<<<(unsigned)((K + 255) / 256), 256, 0, st>>>(c.goff, K, c.t_sorted, c.PS1, c.PS2, c.f_lo[0],
                                                                       c.f_hi[0], c.f_S[0], c.f_Q[0],
                                                                       &c.scalars->ftot[0]);
        c.launches++;
    }
    uint64_t tot = 0;
    CK(cudaMemcpyAsync(&tot, &c.scalars->ftot[0], sizeof(uint64_t), cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
    int cur = 0;
    uint32_t levels = 0;
    while (tot >> 32) {
        const uint64_t C = tot >> 32;
        levels++;
        c.stats.active_rows += tot & 0xFFFFFFFFull;
        const int nxt = cur ^ 1;
        CKS(c.ensure(c.cut, c.cap_cut, sizeof(uint32_t) * C * (kKmMax - 1)));
        CKS(c.ensure(c.km_ngrp, c.cap_km_ngrp, sizeof(uint32_t) * C));
        const uint64_t cap = kk * C;   // at most kk children per cluster
        CKS(c.ensure(c.f_lo[nxt], c.cap_flo[nxt], sizeof(uint32_t) * cap));
        CKS(c.ensure(c.f_hi[nxt], c.cap_fhi[nxt], sizeof(uint32_t) * cap));
        CKS(c.ensure(c.f_S[nxt], c.cap_fS[nxt], sizeof(uint64_t) * cap));
        CKS(c.ensure(c.f_Q[nxt], c.cap_fQ[nxt], sizeof(u128) * cap));
        const int tk_s = c.stage_begin("root_split");
        KmArgs ka{c.f_lo[cur], c.f_hi[cur], &c.scalars->ftot[cur], c.km_dpos, c.km_dP, D, c.km_F,
                  c.km_F + (size_t)(kk + 1) * (D + 1), c.km_arg, kk,
                  c.cut, c.km_ngrp};
        // subproblem lists: at most one per distinct value in flight per round
        const uint64_t rows_l = tot & 0xFFFFFFFFull;
        CKS(c.ensure(c.km_meta, c.cap_km_meta, sizeof(KmMeta) * C));
        // short lists: at most one subproblem per distinct value in flight; long
        // ones: their a ranges (> kKmLong each) overlap only at their ends
        const uint64_t cap_s = rows_l + C + 2, cap_l = rows_l / kKmLong + 2 * C + 2;
        CKS(c.ensure(c.km_sub, c.cap_km_sub, sizeof(KmSub) * 2 * (cap_s + cap_l)));
        KmMeta *meta = (KmMeta *)c.km_meta;
        KmSub *sb = (KmSub *)c.km_sub;
        KmSub *sub[2][2] = {{sb, sb + cap_s}, {sb + 2 * cap_s, sb + 2 * cap_s + cap_l}};   // [class][parity]
        uint32_t *nsub = c.scalars->km_nsub;   // [class * 2 + parity]
        CK(cudaMemsetAsync(nsub, 0, 4 * sizeof(uint32_t), st));
        km_prep_kernel<<<(unsigned)min((C + 7) / 8, (uint64_t)c.sms * 16), 256, 0, st>>>(
            ka, meta, KmLists{{sub[0][0], sub[1][0]}, {nsub + 0, nsub + 2}});
        c.launches++;
        const int depth = 2 + (int)(64 - __builtin_clzll(rows_l + 1));   // rounds: > log2 of the largest d
        for (uint32_t j = 2; j <= kk; j++) {
            if (j > 2) {
                CK(cudaMemsetAsync(nsub, 0, 4 * sizeof(uint32_t), st));
                km_layer_kernel<<<(unsigned)((C + 255) / 256), 256, 0, st>>>(
                    &c.scalars->ftot[cur], meta, j, KmLists{{sub[0][0], sub[1][0]}, {nsub + 0, nsub + 2}});
                c.launches++;
            }
            int sc = 0;
            for (int r = 0; r < depth; r++) {   // empty rounds exit at once (counts read on the device)
                CK(cudaMemsetAsync(nsub + (sc ^ 1), 0, sizeof(uint32_t), st));
                CK(cudaMemsetAsync(nsub + 2 + (sc ^ 1), 0, sizeof(uint32_t), st));
                KmStep ks{ka, meta, {sub[0][sc], sub[1][sc]}, {nsub + sc, nsub + 2 + sc},
                          {sub[0][sc ^ 1], sub[1][sc ^ 1]}, {nsub + (sc ^ 1), nsub + 2 + (sc ^ 1)}, j};
                km_step_block_kernel<<<(unsigned)c.sms * 2, 256, 0, st>>>(ks);
                km_step_warp_kernel<<<(unsigned)c.sms * 16, 256, 0, st>>>(ks);
                c.launches += 2;
                sc ^= 1;
            }
        }
        km_finish_kernel<<<(unsigned)((C + 255) / 256), 256, 0, st>>>(ka, meta);
        c.launches++;
        c.stage_end(tk_s, 12 * rows_l);
        CK(cudaGetLastError());
        const int tk_d = c.stage_begin("root_decide");
        CK(cudaMemsetAsync(&c.scalars->ftot[nxt], 0, sizeof(uint64_t), st));
        KdArgs da{c.f_lo[cur], c.f_hi[cur], c.f_S[cur], c.f_Q[cur], &c.scalars->ftot[cur], c.cut, c.km_ngrp, c.PS1,
                  c.PS2, c.t_sorted, c.flags, c.f_lo[nxt], c.f_hi[nxt], c.f_S[nxt], c.f_Q[nxt],
                  &c.scalars->ftot[nxt], eps, z, k2, clamp, &c.scalars->err};
        kmeans_decide_kernel<<<(unsigned)((C + 127) / 128), 128, 0, st>>>(da);
        c.launches++;
        c.stage_end(tk_d, 96 * C);
        CK(cudaGetLastError());
        CK(cudaMemcpyAsync(&tot, &c.scalars->ftot[nxt], sizeof(uint64_t), cudaMemcpyDeviceToHost, st));
        CK(cudaStreamSynchronize(st));
        cur = nxt;
    }
    c.stats.levels = levels;
    uint32_t err = 0;
    CK(cudaMemcpyAsync(&err, &c.scalars->err, sizeof(uint32_t), cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
    if (err & 8u) return STEM_E_LIMIT;
    return STEM_OK;
}

}  // namespace sr
