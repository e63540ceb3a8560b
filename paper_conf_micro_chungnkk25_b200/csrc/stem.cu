// stem.cu -- steps a5-a8: leaf table, STEM sample sizes (Eq. 6 with the
// corrected numerator, P:L169 + P:L464), Philox sampling with replacement
// (P:L210), weighted-sum extrapolation and predicted bound (Eq. 5).
#include "internal.h"

namespace sr {

constexpr int kThreads = 256;

// ---------------------------------------------------------------- fixed point
// term >= 2^-20 and < 2^100 (R12): value = mant * 2^(exp-1075);
// in units of 2^-72 it is mant << (exp - 1003), spread over 32-bit digits.
__device__ __forceinline__ void fix_digits(double d, uint32_t dig[3], int &q, bool &bad) {
    dig[0] = dig[1] = dig[2] = 0;
    q = 0;
    if (!(d > 0.0)) return;
    const uint64_t bits = (uint64_t)__double_as_longlong(d);
    const int ex = (int)((bits >> 52) & 0x7FF);
    const uint64_t mant = (bits & ((1ull << 52) - 1)) | (1ull << 52);
    const int shift = ex - 1003;
    if (shift < 0 || shift + 53 > 32 * kFixDigits) { bad = true; return; }
    q = shift >> 5;
    const u128 v = (u128)mant << (shift & 31);
    dig[0] = (uint32_t)v;
    dig[1] = (uint32_t)(v >> 32);
    dig[2] = (uint32_t)(v >> 64);
}

// round-to-nearest of sum_j lane[j] 2^(32 j - 72)
__device__ double fix_round(const uint64_t *lane) {
    uint32_t d[kFixDigits + 2];
    u128 carry = 0;
    for (int j = 0; j < kFixDigits; j++) {
        const u128 x = (u128)lane[j] + carry;
        d[j] = (uint32_t)x;
        carry = x >> 32;
    }
    d[kFixDigits] = (uint32_t)carry;
    d[kFixDigits + 1] = (uint32_t)(carry >> 32);
    int top = -1;
    for (int j = kFixDigits + 1; j >= 0; j--)
        if (d[j]) { top = j; break; }
    if (top < 0) return 0.0;
    const int msb = 32 * top + 31 - __clz(d[top]);
    // gather the 64 bits [msb-63, msb]; sticky = any lower bit
    uint64_t word = 0;
    bool sticky = false;
    const int lo_bit = msb - 63;
    for (int b = msb; b >= 0 && b >= lo_bit; b--) word = (word << 1) | ((d[b >> 5] >> (b & 31)) & 1u);
    for (int b = lo_bit - 1; b >= 0 && !sticky; b--) sticky = (d[b >> 5] >> (b & 31)) & 1u;
    const int scale = (lo_bit > 0 ? lo_bit : 0) - kFixLsb;
    if (sticky) word |= 1;
    return __dmul_rn(__ull2double_rn(word), pow2(scale));
}

// ---------------------------------------------------------------- leaf table
// leaf starts = the set bits of the leaf-start bitmap (bit i & 31 of word
// i >> 5); tile = 256 threads x 8 words (65 536 rows), two uint4 per thread
constexpr int kFlagWords = 8;
constexpr uint64_t kFlagTileW = (uint64_t)kThreads * kFlagWords;

__device__ __forceinline__ void flag_words(const uint32_t *f, uint64_t nw, uint64_t w0, uint32_t (&wv)[kFlagWords]) {
    if (w0 + kFlagWords <= nw) {
        const uint4 a = __ldcs(reinterpret_cast<const uint4 *>(f + w0)), b = __ldcs(reinterpret_cast<const uint4 *>(f + w0 + 4));
        wv[0] = a.x; wv[1] = a.y; wv[2] = a.z; wv[3] = a.w; wv[4] = b.x; wv[5] = b.y; wv[6] = b.z; wv[7] = b.w;
    } else {
#pragma unroll
        for (int q = 0; q < kFlagWords; q++) wv[q] = w0 + q < nw ? f[w0 + q] : 0u;
    }
}

__global__ void __launch_bounds__(kThreads) flag_count_kernel(const uint32_t *__restrict__ flags, uint64_t nw,
                                                             uint64_t *__restrict__ tile_cnt) {
    __shared__ uint64_t sm[kThreads / 32 + 1];
    uint32_t wv[kFlagWords];
    flag_words(flags, nw, blockIdx.x * kFlagTileW + (uint64_t)threadIdx.x * kFlagWords, wv);
    uint64_t c = 0;
#pragma unroll
    for (int q = 0; q < kFlagWords; q++) c += __popc(wv[q]);
    uint64_t tot;
    block_excl_scan<uint64_t, kThreads>(c, sm, &tot);
    if (threadIdx.x == 0) tile_cnt[blockIdx.x] = tot;
}

__global__ void __launch_bounds__(kThreads) flag_compact_kernel(const uint32_t *__restrict__ flags, uint64_t nw,
                                                               const uint64_t *__restrict__ tile_off,
                                                               uint32_t *__restrict__ leaf_lo) {
    __shared__ uint64_t sm[kThreads / 32 + 1];
    const uint64_t w0 = blockIdx.x * kFlagTileW + (uint64_t)threadIdx.x * kFlagWords;
    uint32_t wv[kFlagWords];
    flag_words(flags, nw, w0, wv);
    uint64_t c = 0;
#pragma unroll
    for (int q = 0; q < kFlagWords; q++) c += __popc(wv[q]);
    uint64_t tot;
    uint64_t pos = block_excl_scan<uint64_t, kThreads>(c, sm, &tot) + tile_off[blockIdx.x];
#pragma unroll
    for (int q = 0; q < kFlagWords; q++) {
        uint32_t x = wv[q];
        while (x) {
            leaf_lo[pos++] = (uint32_t)((w0 + q) * 32 + (uint32_t)(__ffs(x) - 1));
            x &= x - 1;
        }
    }
}

struct LeafArgs {
    const uint32_t *leaf_lo, *goff, *t;
    const uint64_t *PS1;
    const u128 *PS2;
    uint64_t L, n;
    uint32_t K;
    int scope;
    uint32_t *leaf_kid, *leaf_ord;
    uint64_t *fix_acc;   // [scope==1 ? K : 1][kFixDigits]
    uint64_t *kern_T;    // scope 1
    uint32_t *err;
    const uint32_t *ord_off;   // multi-GPU: ordinal of the kernel's first local leaf (NULL: 0)
};

struct LeafView {
    uint32_t lo, hi;
    uint64_t n, S;
    u128 V;
};

__device__ __forceinline__ LeafView leaf_view(const uint32_t *leaf_lo, uint64_t L, uint64_t N, const uint64_t *PS1,
                                              const u128 *PS2, const uint32_t *t, uint64_t i) {
    LeafView v;
    v.lo = leaf_lo[i];
    v.hi = (i + 1 < L) ? leaf_lo[i + 1] : (uint32_t)N;
    v.n = v.hi - v.lo;
    uint64_t s0, s1;
    u128 q0, q1;
    pref12(PS1, PS2, t, v.lo, s0, q0);
    pref12(PS1, PS2, t, v.hi, s1, q1);
    v.S = s1 - s0;
    const u128 Q = q1 - q0;
    v.V = (u128)v.n * Q - (u128)v.S * v.S;
    return v;
}

// T = sum of all t (exact), from the sampled prefix
__global__ void total_kernel(const uint64_t *PS1, const uint32_t *t, uint64_t n, uint64_t *T) {
    if (threadIdx.x == 0 && blockIdx.x == 0) *T = pref1(PS1, t, n);
}

__global__ void __launch_bounds__(kThreads) leaf_kkt_kernel(LeafArgs a) {
    __shared__ unsigned long long s_acc[kFixDigits];
    if (threadIdx.x < kFixDigits) s_acc[threadIdx.x] = 0;
    __syncthreads();
    const uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    bool bad = false;
    if (i < a.L) {
        const LeafView v = leaf_view(a.leaf_lo, a.L, a.n, a.PS1, a.PS2, a.t, i);
        const uint32_t g = (uint32_t)upper_bound(a.goff, (uint64_t)a.K + 1, v.lo) - 1;
        const uint64_t first = lower_bound(a.leaf_lo, a.L, a.goff[g]);
        a.leaf_kid[i] = g;
        a.leaf_ord[i] = (uint32_t)(i - first) + (a.ord_off ? a.ord_off[g] : 0u);
        if (a.scope != 2) {
            const double mu = __ddiv_rn(rn64(v.S), rn64(v.n));
            const double term = __dsqrt_rn(__dmul_rn(mu, rn128(v.V)));
            uint32_t dig[3];
            int q;
            fix_digits(term, dig, q, bad);
            if (a.scope == 0) {
                for (int j = 0; j < 3; j++)
                    if (dig[j]) atomicAdd(&s_acc[q + j], (unsigned long long)dig[j]);
            } else {
                for (int j = 0; j < 3; j++)
                    if (dig[j]) atomicAdd((unsigned long long *)&a.fix_acc[(uint64_t)g * kFixDigits + q + j],
                                          (unsigned long long)dig[j]);
                atomicAdd((unsigned long long *)&a.kern_T[g], (unsigned long long)v.S);
            }
        }
    }
    if (bad) atomicOr(a.err, 2u);
    __syncthreads();
    if (a.scope == 0 && threadIdx.x < kFixDigits && s_acc[threadIdx.x])
        atomicAdd((unsigned long long *)&a.fix_acc[threadIdx.x], s_acc[threadIdx.x]);
}

// g = Ssum / c with c = (eps T / z)^2 (R10, R11); global: one thread, per kernel: one per kernel
__global__ void kkt_finalize_kernel(const uint64_t *fix_acc, const uint64_t *kern_T, const uint64_t *T,
                                    uint32_t nsets, double eps, double z, double *g_out, double *ssum_out) {
    const uint64_t s = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (s >= nsets) return;
    const double ssum = fix_round(fix_acc + s * kFixDigits);
    const uint64_t Ts = kern_T ? kern_T[s] : *T;
    const double w = __ddiv_rn(__dmul_rn(eps, rn64(Ts)), z);
    const double c = __dmul_rn(w, w);
    g_out[s] = __ddiv_rn(ssum, c);
    if (ssum_out) *ssum_out = ssum;
}

struct MArgs {
    const uint32_t *leaf_lo, *leaf_kid, *t;
    const uint64_t *PS1;
    const u128 *PS2;
    uint64_t L, n;
    int scope, census_cap;
    double k2;
    const double *g;     // [1] or [K]
    uint64_t *m;
    uint8_t *census;
    uint32_t *limit_err;
};

__global__ void __launch_bounds__(kThreads) leaf_m_kernel(MArgs a) {
    const uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= a.L) return;
    const LeafView v = leaf_view(a.leaf_lo, a.L, a.n, a.PS1, a.PS2, a.t, i);
    double m;
    if (v.V == 0) {
        m = 1.0;
    } else if (a.scope == 2) {   // Eq. 3 per leaf
        const double dS = rn64(v.S);
        m = ceil(__dmul_rn(__ddiv_rn(rn128(v.V), __dmul_rn(dS, dS)), a.k2));
    } else {                     // Eq. 6, corrected numerator
        const double mu = __ddiv_rn(rn64(v.S), rn64(v.n));
        const double g = a.scope == 0 ? a.g[0] : a.g[a.leaf_kid[i]];
        m = ceil(__dmul_rn(g, __dsqrt_rn(__ddiv_rn(rn128(v.V), mu))));
    }
    if (m < 1.0) m = 1.0;
    uint8_t cen = 0;
    if (a.census_cap && m >= rn64(v.n)) { m = rn64(v.n); cen = 1; }
    if (!(m < 4294967296.0)) { atomicOr(a.limit_err, 1u); m = 1.0; }
    a.m[i] = (uint64_t)m;
    a.census[i] = cen;
}

// ---------------------------------------------------------------- a7: samples
struct SampleArgs {
    const uint32_t *leaf_lo, *leaf_kid, *leaf_ord;
    const uint64_t *moff, *m;
    const uint8_t *census;
    const uint32_t *t, *row;             // t_sorted; row_sorted (payload) or low row bits (packed)
    uint64_t L, n, S;
    uint32_t key0, key1, kid_base;
    uint32_t *out_row, *out_cluster;
    double *out_weight;
    uint64_t *U;
    // packed sort (sort.cu): the full row is one of pack_h candidates
    // (h << pack_s) | lo; the sort's input columns tell which
    int pack_s;
    uint32_t pack_h;
    const uint32_t *kid_in, *t_in, *row_in;   // sort input (row_in: local -> trace row, or NULL)
    struct Amb *amb;
    uint32_t *amb_count;
};

// a sample whose low row bits match more than one candidate row
struct Amb {
    uint64_t mask;      // candidates h that hold (kernel, t)
    uint32_t s, leaf, pos, lo;
    uint32_t a, b;      // counted range of the run (the shorter side of pos)
    uint32_t side, q;   // side 0: [r0, pos), 1: (pos, r1); q = matches of lo in [a, b)
};
__device__ __forceinline__ uint32_t map_row(const SampleArgs &a, uint32_t r) {
    return a.row_in ? __ldg(a.row_in + r) : r;
}

__global__ void __launch_bounds__(kThreads) sample_kernel(SampleArgs a) {
    const uint64_t s = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (s >= a.S) return;
    // leaf of sample s: s itself while every earlier leaf has m = 1 (the common
    // case: one load), else a binary search over the sample offsets
    uint64_t i = s;
    if (!(s < a.L && a.moff[s] == s)) i = upper_bound(a.moff, a.L, s) - 1;
    const uint64_t j = s - a.moff[i];
    const uint32_t lo = a.leaf_lo[i];
    const uint32_t hi = (i + 1 < a.L) ? a.leaf_lo[i + 1] : (uint32_t)a.n;
    const uint64_t n = hi - lo, m = a.m[i];
    uint64_t pos;
    if (a.census[i]) {
        pos = lo + j;
    } else {
        const U4 x = philox4x32_10(U4{(uint32_t)(j >> 1), a.leaf_ord[i], a.kid_base + a.leaf_kid[i], 0x53544D31u},
                                   a.key0, a.key1);
        const uint64_t r = (j & 1) ? (((uint64_t)x.w << 32) | x.z) : (((uint64_t)x.y << 32) | x.x);
        pos = lo + __umul64hi(r, n);
    }
    SR_DCHECK(i < a.L && j < m && pos >= lo && pos < hi);
    const uint32_t tv = a.t[pos];
    if (a.pack_h == 0) {
        a.out_row[s] = a.row[pos];
    } else {
        const uint32_t low = a.row[pos];
        if (a.pack_h == 1) {
            a.out_row[s] = map_row(a, low);
        } else {
            // rows with the same (kernel, t) are in ascending row order in the
            // sorted run; the candidates (h << s) | low that hold (kernel, t)
            const uint32_t k = a.leaf_kid[i];
            uint64_t mask = 0;
            for (uint32_t h0 = 0; h0 < a.pack_h; h0 += 16) {   // 16 candidates' times in flight
                uint32_t tw[16];
#pragma unroll
                for (int u = 0; u < 16; u++) {
                    const uint64_t r = ((uint64_t)(h0 + u) << a.pack_s) | low;
                    const bool ok = h0 + u < a.pack_h && r < a.n;
                    tw[u] = ok ? __ldg(a.t_in + r) : ~tv;   // never equal to tv
                }
                // the kernel id only where the time matches (most candidates differ in t)
#pragma unroll
                for (int u = 0; u < 16; u++)
                    if (tw[u] == tv && __ldg(a.kid_in + (((uint64_t)(h0 + u) << a.pack_s) | low)) == k)
                        mask |= 1ull << (h0 + u);
            }
            if (__popcll(mask) == 1) {
                a.out_row[s] = map_row(a, (uint32_t)(((uint64_t)(__ffsll(mask) - 1) << a.pack_s) | low));
            } else {   // resolved by resolve_kernel: which of the matches sits at pos
                const uint32_t e = atomicAdd(a.amb_count, 1u);
                SR_DCHECK(e < a.S && __popcll(mask) >= 1);
                a.amb[e] = Amb{mask, (uint32_t)s, (uint32_t)i, (uint32_t)pos, low};
            }
        }
    }
    a.out_cluster[s] = (uint32_t)i;
    a.out_weight[s] = __ddiv_rn(rn64(n), rn64(m));
    atomicAdd((unsigned long long *)&a.U[i], (unsigned long long)tv);
}

// Ambiguous sample at pos in the run [r0, r1) of equal (kernel, t): the run
// lists the matching rows in ascending order and the low bits of each element
// are known, so the sample is the q-th (ascending) of its candidates, where q
// counts the run's elements before pos with the same low bits (or, counting
// the shorter side, M - 1 - the elements after pos).  Three steps: locate the
// run and the side to count, count it in 64k-element chunks over the whole
// grid, pick the candidate.
constexpr uint32_t kAmbChunk = 1u << 16;

// (the ambiguous-sample count na is read on the device: grids are sized for
// every sample, entries past na get no chunks; no host round trip)
__global__ void __launch_bounds__(kThreads) resolve_locate_kernel(SampleArgs a, const uint32_t *nap, uint64_t *nch) {
    const uint32_t e = blockIdx.x * blockDim.x + threadIdx.x;
    if (e >= a.S) return;
    if (e >= *nap) { nch[e] = 0; return; }
    Amb &en = a.amb[e];
    const uint32_t tv = a.t[en.pos];
    const uint32_t lo = a.leaf_lo[en.leaf];
    const uint32_t hi = (en.leaf + 1 < a.L) ? a.leaf_lo[en.leaf + 1] : (uint32_t)a.n;
    const uint32_t r0 = lo + (uint32_t)lower_bound(a.t + lo, (uint64_t)(en.pos - lo), tv);
    const uint32_t r1 = en.pos + 1 + (uint32_t)upper_bound(a.t + en.pos + 1, (uint64_t)(hi - en.pos - 1), tv);
    if (en.pos - r0 <= r1 - en.pos - 1) { en.a = r0; en.b = en.pos; en.side = 0; }
    else { en.a = en.pos + 1; en.b = r1; en.side = 1; }
    en.q = 0;
    nch[e] = (en.b - en.a + kAmbChunk - 1) / kAmbChunk;
}

__global__ void __launch_bounds__(kThreads) resolve_count_kernel(SampleArgs a, uint32_t na, const uint64_t *choff,
                                                                 const uint64_t *total) {
    __shared__ uint32_t s_cnt[kThreads / 32];
    const uint64_t nc = *total;
    for (uint64_t c = blockIdx.x; c < nc; c += gridDim.x) {
        const uint32_t e = (uint32_t)(upper_bound(choff, (uint64_t)na, c) - 1);
        const Amb &en = a.amb[e];
        const uint32_t x0 = en.a + (uint32_t)(c - choff[e]) * kAmbChunk;
        const uint32_t x1 = min(en.b, x0 + kAmbChunk);
        const uint32_t v = en.lo;
        uint32_t q = 0;
        const uint32_t v0 = min(x1, (x0 + 3) & ~3u), v1 = max(v0, x1 & ~3u);
        for (uint32_t x = x0 + threadIdx.x; x < v0; x += blockDim.x) q += __ldcs(a.row + x) == v;
        for (uint32_t x = v1 + threadIdx.x; x < x1; x += blockDim.x) q += __ldcs(a.row + x) == v;
        const uint4 *p4 = reinterpret_cast<const uint4 *>(a.row + v0);
        const uint32_t n4 = (v1 - v0) / 4;
#pragma unroll 4
        for (uint32_t x = threadIdx.x; x < n4; x += blockDim.x) {
            const uint4 w = __ldcs(p4 + x);
            q += (w.x == v) + (w.y == v) + (w.z == v) + (w.w == v);
        }
        for (int o = 16; o; o >>= 1) q += __shfl_xor_sync(0xffffffffu, q, o);
        if ((threadIdx.x & 31) == 0) s_cnt[threadIdx.x >> 5] = q;
        __syncthreads();
        if (threadIdx.x == 0) {
            uint32_t qq = 0;
            for (int w = 0; w < kThreads / 32; w++) qq += s_cnt[w];
            if (qq) atomicAdd(&a.amb[e].q, qq);
        }
        __syncthreads();
    }
}

__global__ void __launch_bounds__(kThreads) resolve_final_kernel(SampleArgs a, const uint32_t *nap) {
    const uint32_t e = blockIdx.x * blockDim.x + threadIdx.x;
    if (e >= *nap) return;
    const Amb en = a.amb[e];
    const uint32_t M = (uint32_t)__popcll(en.mask);
    uint32_t idx = en.side ? M - 1 - en.q : en.q;
    uint64_t mk = en.mask;
    for (uint32_t b = 0; b < idx && mk; b++) mk &= mk - 1;   // drop the idx lowest matches
    const uint32_t h = mk ? (uint32_t)(__ffsll(mk) - 1) : 0u;
    a.out_row[en.s] = map_row(a, (uint32_t)(((uint64_t)h << a.pack_s) | en.lo));
}

// ---------------------------------------------------------------- a8: estimate
// deterministic block sum (fixed tree for a fixed launch shape)
__device__ __forceinline__ double block_sum(double v, double *sm) {
    for (int o = 16; o; o >>= 1) v = __dadd_rn(v, __shfl_xor_sync(0xffffffffu, v, o));
    const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
    __syncthreads();
    if (lane == 0) sm[w] = v;
    __syncthreads();
    double r = 0.0;
    if (threadIdx.x == 0)
        for (int k = 0; k < (int)(blockDim.x >> 5); k++) r = __dadd_rn(r, sm[k]);
    return r;   // valid in thread 0
}

struct EstArgs {
    const uint32_t *leaf_lo, *t;
    const uint64_t *PS1;
    const u128 *PS2;
    const uint64_t *m, *U;
    uint64_t L, n;
    uint64_t *sum_q;
    double *part;   // [blocks][2]
};

__global__ void __launch_bounds__(kThreads) estimate_kernel(EstArgs a) {
    __shared__ double sm[kThreads / 32];
    __shared__ unsigned long long s_q[kThreads / 32];
    const uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    double frac = 0.0, var = 0.0;
    uint64_t q = 0;
    if (i < a.L) {
        const LeafView v = leaf_view(a.leaf_lo, a.L, a.n, a.PS1, a.PS2, a.t, i);
        const uint64_t m = a.m[i];
        const u128 num = (u128)v.n * a.U[i];
        uint64_t r;
        if ((uint64_t)(num >> 64) == 0) {   // the common case (m = 1: U < 2^32): 64-bit division
            q = (uint64_t)num / m;
            r = (uint64_t)num - q * m;
        } else {
            q = (uint64_t)(num / m);
            r = (uint64_t)(num % m);
        }
        frac = __ddiv_rn(rn64(r), rn64(m));
        var = __ddiv_rn(rn128(v.V), rn64(m));
    }
    // sum_i q_i: one atomic per block (exact integer, any order)
    for (int o = 16; o; o >>= 1) q += __shfl_xor_sync(0xffffffffu, q, o);
    if ((threadIdx.x & 31) == 0) s_q[threadIdx.x >> 5] = q;
    const double f = block_sum(frac, sm);
    const double vv = block_sum(var, sm);
    if (threadIdx.x == 0) {
        unsigned long long bq = 0;
        for (int w = 0; w < kThreads / 32; w++) bq += s_q[w];
        if (bq) atomicAdd((unsigned long long *)a.sum_q, bq);
        a.part[2 * blockIdx.x] = f;
        a.part[2 * blockIdx.x + 1] = vv;
    }
}

struct MetArgs {
    const uint32_t *out_row;
    const double *out_weight;
    const double *metrics;
    uint64_t n, S;
    uint32_t nm;
    double *part;   // [blocks][nm]
};

__global__ void __launch_bounds__(kThreads) metric_kernel(MetArgs a) {
    __shared__ double sm[kThreads / 32];
    const uint64_t s = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    for (uint32_t c = 0; c < a.nm; c++) {
        double v = 0.0;
        if (s < a.S) v = __dmul_rn(a.out_weight[s], a.metrics[(uint64_t)c * a.n + a.out_row[s]]);
        const double r = block_sum(v, sm);
        if (threadIdx.x == 0) a.part[(uint64_t)blockIdx.x * a.nm + c] = r;
    }
}

// sums block partials column by column in block order (deterministic)
__global__ void reduce_cols_kernel(const double *part, uint64_t blocks, uint32_t cols, double *out) {
    __shared__ double sm[kThreads / 32];
    for (uint32_t c = 0; c < cols; c++) {
        double v = 0.0;
        for (uint64_t b = threadIdx.x; b < blocks; b += blockDim.x) v = __dadd_rn(v, part[b * cols + c]);
        const double r = block_sum(v, sm);
        if (threadIdx.x == 0) out[c] = r;
    }
}

// est = rn(sum_i q_i) + sum_i rn(r_i)/m_i ; bound = z sqrt(sum_i V_i/m_i) / T  (R16, R17)
__global__ void est_finalize_kernel(const uint64_t *sum_q, const double *red, const uint64_t *T, double z,
                                    double *out) {
    out[0] = __dadd_rn(rn64(*sum_q), red[0]);
    out[1] = (*T == 0) ? 0.0 : __ddiv_rn(__dmul_rn(z, __dsqrt_rn(red[1])), rn64(*T));
}

__global__ void pack_kernel(const uint32_t *leaf_lo, const uint32_t *leaf_kid, const uint32_t *leaf_ord,
                            const uint64_t *PS1, const u128 *PS2, const uint32_t *t, const uint64_t *m,
                            const uint8_t *census, uint64_t L, uint64_t n, uint32_t kid_base, stem_cluster *out) {
    const uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= L) return;
    const LeafView v = leaf_view(leaf_lo, L, n, PS1, PS2, t, i);
    stem_cluster c;
    c.kernel_id = kid_base + leaf_kid[i];
    c.ordinal = leaf_ord[i];
    c.lo_ns = t[v.lo];
    c.hi_ns = t[v.hi - 1];
    c.n = v.n;
    c.sum_ns = v.S;
    const double dn = rn64(v.n);
    c.mean_ns = __ddiv_rn(rn64(v.S), dn);
    c.std_ns = __ddiv_rn(__dsqrt_rn(rn128(v.V)), dn);
    c.m = m[i];
    c.census = census[i];
    c.reserved = 0;
    out[i] = c;
}

// ---------------------------------------------------------------- driver
static unsigned blocks_for(uint64_t n) { return (unsigned)((n + kThreads - 1) / kThreads); }

// In multi-GPU runs every stretch of local work between two collectives is one
// segment: its status is agreed across ranks (dist_checkpoint) before the next
// collective, so a rank-local failure (allocation, CUDA) makes every rank
// return the same error instead of leaving peers blocked in a collective.
int leaves_and_plan(Ctx &c, uint64_t n, uint32_t K, const double *metrics, uint32_t nm, double eps, double z,
                    double k2, const stem_opts &o, const uint32_t *tr_kid, const uint32_t *tr_t, uint64_t tr_n) {
    cudaStream_t st = c.stream;
    uint64_t L = 0;
    const uint32_t nsets = o.scope == 1 ? K : 1;
    // ---- segment 1: leaf table (a5) and the exact KKT partials (a6)
    CKS(dist_checkpoint(c, [&]() -> int {
        // a5: leaf starts = group starts U accepted cuts, in row order = canonical (kernel, lo) order
        CKS(c.ensure(c.scan_scratch, c.cap_scan, (scan_tiles(n) + 1) * sizeof(uint64_t)));
        CKS(c.ensure(c.leaf_lo, c.cap_leaf_lo, sizeof(uint32_t) * (n + 1)));
        const int tk_leaf = c.stage_begin("leaf_table");
        {
            const uint64_t nw = (n + 31) / 32, nt = (nw + kFlagTileW - 1) / kFlagTileW;   // bits >= n are never set
            CKS(c.ensure(c.leaf_moff, c.cap_leaf_moff, sizeof(uint64_t) * (nt + 1)));   // tile counts (scratch)
            uint64_t *tcnt = c.leaf_moff;
            if (nt) flag_count_kernel<<<(unsigned)nt, kThreads, 0, st>>>(c.flags, nw, tcnt);
            exclusive_scan<uint64_t>([tcnt] __device__(uint64_t i) -> uint64_t { return tcnt[i]; },
                                     [tcnt] __device__(uint64_t i, uint64_t pre, uint64_t) { tcnt[i] = pre; }, nt,
                                     (uint64_t *)c.scan_scratch, &c.scalars->n_leaves, st, &c.launches);
            if (nt) flag_compact_kernel<<<(unsigned)nt, kThreads, 0, st>>>(c.flags, nw, tcnt, c.leaf_lo);
            c.launches += 2;
            CK(cudaGetLastError());
        }
        c.stage_end(tk_leaf, 2 * 4 * (n / 32 + 1));
        CK(cudaMemcpyAsync(&L, &c.scalars->n_leaves, sizeof(uint64_t), cudaMemcpyDeviceToHost, st));
        CKS(sync_stream(c));
        c.n_leaves = L;
        CKS(c.ensure(c.leaf_m, c.cap_leaf_m, sizeof(uint64_t) * (L + 1)));
        CKS(c.ensure(c.leaf_moff, c.cap_leaf_moff, sizeof(uint64_t) * (L + 1)));
        CKS(c.ensure(c.leaf_U, c.cap_leaf_U, sizeof(uint64_t) * (L + 1)));
        CKS(c.ensure(c.leaf_census, c.cap_leaf_census, L + 1));
        CKS(c.ensure(c.leaf_kid, c.cap_leaf_kid, sizeof(uint32_t) * (L + 1)));
        CKS(c.ensure(c.leaf_ord, c.cap_leaf_ord, sizeof(uint32_t) * (L + 1)));
        CKS(c.ensure(c.fix_acc, c.cap_fix, sizeof(uint64_t) * kFixDigits * nsets));
        CKS(c.ensure(c.kern_T, c.cap_kern_T, sizeof(uint64_t) * nsets));
        CKS(c.ensure(c.kern_g, c.cap_kern_g, sizeof(double) * nsets));
        CK(cudaMemsetAsync(c.fix_acc, 0, sizeof(uint64_t) * kFixDigits * nsets, st));
        CK(cudaMemsetAsync(c.kern_T, 0, sizeof(uint64_t) * nsets, st));
        CK(cudaMemsetAsync(c.leaf_U, 0, sizeof(uint64_t) * (L + 1), st));
        return STEM_OK;
    }()));
    uint32_t *leaf_kid = c.leaf_kid, *leaf_ord = c.leaf_ord;

    const int tk_kkt = c.stage_begin("stem_sizes");
    CKS(dist_checkpoint(c, [&]() -> int {
        if (n) {
            total_kernel<<<1, 32, 0, st>>>(c.PS1, c.t_sorted, n, &c.scalars->T);
            c.launches++;
        } else {
            CK(cudaMemsetAsync(&c.scalars->T, 0, sizeof(uint64_t), st));
        }
        LeafArgs la{c.leaf_lo, c.goff, c.t_sorted, c.PS1, c.PS2, L, n, K, o.scope, leaf_kid, leaf_ord,
                    c.fix_acc, c.kern_T, &c.scalars->err, c.ord_off};
        if (L) leaf_kkt_kernel<<<blocks_for(L), kThreads, 0, st>>>(la);
        c.launches++;
        CK(cudaGetLastError());
        return STEM_OK;
    }()));
    if (c.comm) {   // multi-GPU: T and the exact Ssum digits are sums over every rank's leaves
        uint64_t *r7 = c.scalars->red7;
        CK(cudaMemcpyAsync(r7, &c.scalars->T, sizeof(uint64_t), cudaMemcpyDeviceToDevice, st));
        CK(cudaMemcpyAsync(r7 + 1, c.fix_acc, sizeof(uint64_t) * kFixDigits, cudaMemcpyDeviceToDevice, st));
        CKS(dist_allreduce_u64(c, r7, o.scope == 0 ? 1 + kFixDigits : 1));
        CK(cudaMemcpyAsync(&c.scalars->T, r7, sizeof(uint64_t), cudaMemcpyDeviceToDevice, st));
        if (o.scope == 0)
            CK(cudaMemcpyAsync(c.fix_acc, r7 + 1, sizeof(uint64_t) * kFixDigits, cudaMemcpyDeviceToDevice, st));
    }
    // ---- segment 2: g per set, m_i, sample offsets
    CKS(dist_checkpoint(c, [&]() -> int {
        if (o.scope == 0)
            kkt_finalize_kernel<<<1, 32, 0, st>>>(c.fix_acc, nullptr, &c.scalars->T, 1, eps, z, c.kern_g,
                                                  &c.scalars->ssum);
        else if (o.scope == 1 && K)
            kkt_finalize_kernel<<<blocks_for(K), kThreads, 0, st>>>(c.fix_acc, c.kern_T, nullptr, K, eps, z, c.kern_g,
                                                                   nullptr);
        if (o.scope != 2) c.launches++;
        MArgs ma{c.leaf_lo, leaf_kid, c.t_sorted, c.PS1, c.PS2, L, n, o.scope, o.census_cap, k2, c.kern_g,
                 c.leaf_m, c.leaf_census, &c.scalars->limit_err};
        if (L) leaf_m_kernel<<<blocks_for(L), kThreads, 0, st>>>(ma);
        c.launches++;
        CK(cudaGetLastError());
        const uint64_t *m = c.leaf_m;
        uint64_t *moff = c.leaf_moff;
        exclusive_scan<uint64_t>([m] __device__(uint64_t i) -> uint64_t { return m[i]; },
                                 [moff] __device__(uint64_t i, uint64_t pre, uint64_t) { moff[i] = pre; }, L,
                                 (uint64_t *)c.scan_scratch, &c.scalars->total_m, st, &c.launches);
        CK(cudaGetLastError());
        return STEM_OK;
    }()));
    c.stage_end(tk_kkt, 64 * L);
    uint64_t S_global = 0;
    if (c.comm) {
        uint64_t *r7 = c.scalars->red7;
        CK(cudaMemcpyAsync(r7, &c.scalars->total_m, sizeof(uint64_t), cudaMemcpyDeviceToDevice, st));
        CK(cudaMemsetAsync(r7 + 1, 0, sizeof(uint64_t), st));
        CK(cudaMemcpyAsync(r7 + 1, &c.scalars->limit_err, sizeof(uint32_t), cudaMemcpyDeviceToDevice, st));
        CKS(dist_allreduce_u64(c, r7, 2));
        uint64_t h2[2];
        CK(cudaMemcpyAsync(h2, r7, sizeof(h2), cudaMemcpyDeviceToHost, st));
        CKS(sync_stream(c));
        if (h2[1] || h2[0] >= (1ull << 32)) return STEM_E_LIMIT;   // identical on every rank
        S_global = h2[0];
    }
    // ---- segment 3: samples (a7) and the local estimate partials (a8)
    uint64_t S = 0;
    uint32_t n_amb = 0;
    const uint64_t eb = blocks_for(L);
    double *part_est = nullptr, *part_met = nullptr, *red_out = nullptr;
    uint64_t mb = 0;
    int tk_est = -1;
    uint32_t *h_row = nullptr, *h_scl = nullptr;   // the early host plan's sample arrays
    double *h_w = nullptr;
    CKS(dist_checkpoint(c, [&]() -> int {
        DevScalars hs;
        CK(cudaMemcpyAsync(&hs, c.scalars, sizeof(DevScalars), cudaMemcpyDeviceToHost, st));
        CKS(sync_stream(c));
        if (hs.err & 2) return STEM_E_CUDA;
        if (hs.limit_err || hs.total_m >= (1ull << 32)) return STEM_E_LIMIT;
        S = hs.total_m;
        c.n_samples = S;
        c.T = hs.T;
        c.stats.ssum = o.scope == 0 ? hs.ssum : 0.0;
        c.n_samples_global = c.comm ? S_global : S;

        CKS(c.ensure(c.out_row, c.cap_out_row, sizeof(uint32_t) * (S + 1)));
        CKS(c.ensure(c.out_cluster, c.cap_out_cluster, sizeof(uint32_t) * (S + 1)));
        CKS(c.ensure(c.out_weight, c.cap_out_weight, sizeof(double) * (S + 1)));
        // packed sort: ambiguous-sample entries, their chunk counts/offsets, scan scratch
        const size_t amb_bytes = sizeof(Amb) * (S + 1), nch_bytes = sizeof(uint64_t) * (S + 1);
        if (c.pack_h > 1) CKS(c.ensure(c.amb, c.cap_amb, amb_bytes + 2 * nch_bytes + (scan_tiles(S + 1) + 2) * 16));
        c.early_packed = false;
        static const bool early_on = !(getenv("STEMROOT_EARLY_PLAN") && getenv("STEMROOT_EARLY_PLAN")[0] == '0');
        if (c.want_host && !c.comm && L && S && early_on) {
            // the caller's plan block now: the cluster records are packed here (they
            // need only m) and copied to it on dstream while the samples are drawn
            stem_cluster *h_cl = nullptr;
            CKS(plan_block_begin(c, L, S, nm, &h_cl, &h_row, &h_scl, &h_w));
            if (!c.dstream) {
                CK(cudaStreamCreateWithFlags(&c.dstream, cudaStreamNonBlocking));
                CK(cudaEventCreateWithFlags(&c.ev_pack, cudaEventDisableTiming));
                CK(cudaEventCreateWithFlags(&c.ev_d2h, cudaEventDisableTiming));
            }
            CKS(c.ensure(c.out_clusters, c.cap_out_cl, sizeof(stem_cluster) * (L + 1)));
            const int tk_pack = c.stage_begin("pack");
            pack_kernel<<<blocks_for(L), kThreads, 0, st>>>(c.leaf_lo, leaf_kid, leaf_ord, c.PS1, c.PS2, c.t_sorted,
                                                            c.leaf_m, c.leaf_census, L, n, c.kid_base, c.out_clusters);
            c.launches++;
            c.stage_end(tk_pack, 88 * L);
            CK(cudaGetLastError());
            CK(cudaEventRecord(c.ev_pack, st));
            CK(cudaStreamWaitEvent(c.dstream, c.ev_pack, 0));
            CK(cudaMemcpyAsync(h_cl, c.out_clusters, sizeof(stem_cluster) * L, cudaMemcpyDeviceToHost, c.dstream));
            c.early_packed = true;
        }
        SampleArgs sa{c.leaf_lo, leaf_kid, leaf_ord, c.leaf_moff, c.leaf_m, c.leaf_census, c.t_sorted,
                      c.row_sorted, L, n, S, (uint32_t)o.seed, (uint32_t)(o.seed >> 32), c.kid_base, c.out_row,
                      c.out_cluster, c.out_weight, c.leaf_U, c.pack_s, c.pack_h, c.sort_kid, c.sort_t,
                      c.sort_row_in, (Amb *)c.amb, &c.scalars->amb_count};
        const int tk_smp = c.stage_begin("samples");
        CK(cudaMemsetAsync(&c.scalars->amb_count, 0, sizeof(uint32_t), st));
        if (S) sample_kernel<<<blocks_for(S), kThreads, 0, st>>>(sa);
        c.launches += S ? 1 : 0;
        if (S && c.pack_h > 1) {   // ambiguous samples, counted on the device (no host round trip)
            const uint32_t *nap = &c.scalars->amb_count;
            uint64_t *nch = (uint64_t *)((char *)c.amb + amb_bytes), *choff = nch + (S + 1), *scr = choff + (S + 1);
            uint64_t *tot = &c.scalars->scan_total64;
            resolve_locate_kernel<<<blocks_for(S), kThreads, 0, st>>>(sa, nap, nch);
            exclusive_scan<uint64_t>([nch] __device__(uint64_t i) -> uint64_t { return nch[i]; },
                                     [choff] __device__(uint64_t i, uint64_t pre, uint64_t) { choff[i] = pre; },
                                     S, scr, tot, st, &c.launches);
            resolve_count_kernel<<<4 * c.sms, kThreads, 0, st>>>(sa, (uint32_t)S, choff, tot);
            resolve_final_kernel<<<blocks_for(S), kThreads, 0, st>>>(sa, nap);
            c.launches += 3;
        }
        c.stage_end(tk_smp, 40 * S);
        CK(cudaGetLastError());
        if (c.early_plan) {   // the samples' host copies, beside the estimate
            CK(cudaEventRecord(c.ev_d2h, st));
            CK(cudaStreamWaitEvent(c.dstream, c.ev_d2h, 0));
            CK(cudaMemcpyAsync(h_row, c.out_row, sizeof(uint32_t) * S, cudaMemcpyDeviceToHost, c.dstream));
            CK(cudaMemcpyAsync(h_scl, c.out_cluster, sizeof(uint32_t) * S, cudaMemcpyDeviceToHost, c.dstream));
            CK(cudaMemcpyAsync(h_w, c.out_weight, sizeof(double) * S, cudaMemcpyDeviceToHost, c.dstream));
        }

        // a8: estimate, bound, metrics (deterministic block partials)
        mb = blocks_for(S);
        const uint64_t part_cols = 2 + (uint64_t)nm;
        const uint64_t part_doubles = 2 * eb + mb * (nm ? nm : 1) + part_cols + 16;
        CKS(c.ensure(c.red_part, c.cap_red, sizeof(double) * part_doubles));
        part_est = c.red_part;
        part_met = c.red_part + 2 * eb;
        red_out = part_met + mb * (nm ? nm : 1);
        CK(cudaMemsetAsync(&c.scalars->sum_q, 0, sizeof(uint64_t), st));
        tk_est = c.stage_begin("estimate");
        EstArgs ea{c.leaf_lo, c.t_sorted, c.PS1, c.PS2, c.leaf_m, c.leaf_U, L, n, &c.scalars->sum_q, part_est};
        if (eb) estimate_kernel<<<(unsigned)eb, kThreads, 0, st>>>(ea);
        reduce_cols_kernel<<<1, kThreads, 0, st>>>(part_est, eb, 2, red_out);
        c.launches += 2;
        CK(cudaGetLastError());
        return STEM_OK;
    }()));
    if (c.comm) {
        CKS(dist_allreduce_u64(c, &c.scalars->sum_q, 1));
        CKS(dist_allreduce_f64(c, red_out, 2));
        if (nm) CKS(dist_metric_sums(c, metrics, nm, S, red_out + 2));
    } else if (nm && S) {
        MetArgs ma2{c.out_row, c.out_weight, metrics, n, S, nm, part_met};
        metric_kernel<<<(unsigned)mb, kThreads, 0, st>>>(ma2);
        reduce_cols_kernel<<<1, kThreads, 0, st>>>(part_met, mb, nm, red_out + 2);
        c.launches += 2;
    }
    c.stage_end(tk_est, 56 * L + 12 * S * nm);
    // ---- segment 4: cluster records, final scalars
    CKS(dist_checkpoint(c, [&]() -> int {
        if (!c.early_packed) {
            CKS(c.ensure(c.out_clusters, c.cap_out_cl, sizeof(stem_cluster) * (L + 1)));
            const int tk_pack = c.stage_begin("pack");
            if (L)
                pack_kernel<<<blocks_for(L), kThreads, 0, st>>>(c.leaf_lo, leaf_kid, leaf_ord, c.PS1, c.PS2,
                                                                c.t_sorted, c.leaf_m, c.leaf_census, L, n, c.kid_base,
                                                                c.out_clusters);
            c.launches++;
            c.stage_end(tk_pack, 88 * L);
            CK(cudaGetLastError());
        }
        double *est_out = red_out + 2 + nm;
        est_finalize_kernel<<<1, 1, 0, st>>>(&c.scalars->sum_q, red_out, &c.scalars->T, z, est_out);
        c.launches++;
        CK(cudaGetLastError());
        double red[2 + 64 + 2];
        CK(cudaMemcpyAsync(red, red_out, sizeof(double) * (2 + nm + 2), cudaMemcpyDeviceToHost, st));
        if (c.pack_h > 1) CK(cudaMemcpyAsync(&n_amb, &c.scalars->amb_count, sizeof(uint32_t), cudaMemcpyDeviceToHost, st));
        CKS(sync_stream(c));
        c.est_total = red[2 + nm];
        c.bound = red[2 + nm + 1];
        for (uint32_t k = 0; k < nm; k++) c.host_est_metric[k] = (S || c.comm) ? red[2 + k] : 0.0;
        c.stats.n_clusters = L;
        c.stats.n_samples = S;
        c.stats.ambiguous_samples = n_amb;
        c.have_mbounds = false;
        if (o.metric_bounds && nm && !c.comm) {   // multi-GPU: metric_bounds_dist after the plan is gathered
            const int tk_mb = c.stage_begin("metric_bounds");
            CKS(metric_bounds_local(c, L, K, n, tr_kid, tr_t, metrics, tr_n, nm, z));
            c.stage_end(tk_mb, (16 + 16 * (uint64_t)nm) * tr_n);
            c.have_mbounds = true;
        }
        return STEM_OK;
    }()));
    return STEM_OK;
}

}  // namespace sr
