// common.cuh -- shared device helpers of the STEM+ROOT CUDA library (sm_100a).
// Exact integer arithmetic (u128/u256), correctly rounded conversions, the
// split-candidate order, Philox4x32-10, block-level scans.  No oracle code.
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

typedef unsigned __int128 u128;
typedef __int128 i128;

// Device-side bounds checks of the checked build (-DSR_CHECK: tests/test_gpu_checked.py,
// the stand-in for compute-sanitizer's memcheck where the GPU pool disables it).
// A failed check prints its site and traps (the context dies, the call fails loudly).
#ifdef SR_CHECK
#include <cstdio>
#define SR_DCHECK(cond)                                                                  \
    do {                                                                                 \
        if (!(cond)) {                                                                   \
            printf("SR_CHECK failed at %s:%d: %s (block %d thread %d)\n", __FILE__, __LINE__, #cond, \
                   (int)blockIdx.x, (int)threadIdx.x);                                   \
            __trap();                                                                    \
        }                                                                                \
    } while (0)
#else
#define SR_DCHECK(cond) do { } while (0)
#endif

namespace sr {

constexpr int kWarp = 32;

// ---------------------------------------------------------------- conversions
// Round-to-nearest-even conversion of an exact u64 / u128 to double.
__device__ __forceinline__ double rn64(uint64_t v) { return __ull2double_rn(v); }

__device__ __forceinline__ double pow2(int e) {  // exact 2^e, -1022 <= e <= 1023
    return __longlong_as_double((long long)(1023 + e) << 52);
}

__device__ __forceinline__ double rn128(u128 v) {
    const uint64_t hi = (uint64_t)(v >> 64);
    if (hi == 0) return __ull2double_rn((uint64_t)v);
    const int lz = __clzll(hi);
    const u128 s = v << lz;                       // MSB now at bit 127
    uint64_t top = (uint64_t)(s >> 64);
    top |= (uint64_t)((uint64_t)s != 0);          // sticky: 11 guard bits below the 53 kept
    return __dmul_rn(__ull2double_rn(top), pow2(64 - lz));
}

// ---------------------------------------------------------------- u256 products
struct U256 { uint64_t w[4]; };

__device__ __forceinline__ void mac(uint64_t a, uint64_t b, uint64_t &lo, uint64_t &hi) {
    lo = a * b;
    hi = __umul64hi(a, b);
}

// (a1:a0)^2 * p for |D| = (a1:a0) < 2^96 and p < 2^64; the product is < 2^256.
__device__ __forceinline__ U256 sq_times(u128 d, uint64_t p) {
    const uint64_t a0 = (uint64_t)d, a1 = (uint64_t)(d >> 64);
    // s = d^2 as 3 limbs (a1 < 2^32 so d^2 < 2^192)
    uint64_t l00, h00, l01, h01, l11, h11;
    mac(a0, a0, l00, h00);
    mac(a0, a1, l01, h01);
    mac(a1, a1, l11, h11);
    // d^2 = l00 + (h00 + 2*l01) 2^64 + (2*h01 + l11) 2^128 + h11 2^192 (h11 = 0)
    u128 mid = (u128)h00 + ((u128)l01 << 1);
    const uint64_t s0 = l00, s1 = (uint64_t)mid;
    u128 top = (mid >> 64) + ((u128)h01 << 1) + l11;
    const uint64_t s2 = (uint64_t)top;
    // times p
    U256 r;
    uint64_t lo, hi;
    mac(s0, p, lo, hi);
    r.w[0] = lo;
    u128 acc = (u128)hi;
    mac(s1, p, lo, hi);
    acc += lo;
    r.w[1] = (uint64_t)acc;
    acc = (acc >> 64) + hi;
    mac(s2, p, lo, hi);
    acc += lo;
    r.w[2] = (uint64_t)acc;
    acc = (acc >> 64) + hi;
    r.w[3] = (uint64_t)acc;
    return r;
}

__device__ __forceinline__ int cmp256(const U256 &a, const U256 &b) {
#pragma unroll
    for (int i = 3; i >= 0; i--)
        if (a.w[i] != b.w[i]) return a.w[i] < b.w[i] ? -1 : 1;
    return 0;
}

// ---------------------------------------------------------------- split candidates
// Candidate cut k of a cluster: score = D^2 / p, D = n*S_L - S*k (<= 0 for
// sorted data, |D| < 2^96), p = k (n - k).  x = fp64 |D|^2 is the filter
// value (relative error < 2^-50); SL = S_L(k) travels to the decision.
struct Cand {
    double x;       // ~ |D|^2
    double dp;      // ~ p
    uint64_t dlo;   // |D| bits 0..63
    uint64_t p;
    uint64_t SL;
    uint32_t dhi;   // |D| bits 64..95
    uint32_t k;     // 0 = no candidate
};

__device__ __forceinline__ Cand no_cand() {
    Cand c;
    c.x = 0.0;
    c.dp = 0.0;
    c.dlo = 0;
    c.p = 0;
    c.SL = 0;
    c.dhi = 0;
    c.k = 0;
    return c;
}

__device__ __forceinline__ u128 cand_absD(const Cand &c) { return ((u128)c.dhi << 64) | c.dlo; }

// fp64 approximation of |D| = hi:lo (hi < 2^32), relative error <= 2^-52
__device__ __forceinline__ double approx_d(uint32_t hi, uint64_t lo) {
    return __fma_rn(__uint2double_rn(hi), 0x1p64, __ull2double_rn(lo));
}

// Exact comparison D_a^2 p_b vs D_b^2 p_a (both < 2^256): -1, 0, +1
__device__ __forceinline__ int exact_cmp(const Cand &a, const Cand &b) {
    return cmp256(sq_times(cand_absD(a), b.p), sq_times(cand_absD(b), a.p));
}

// Exact strict total order (R5): larger score first, ties -> smaller k.
// x_a * dp_b vs x_b * dp_a in fp64 (each side within 2^-49 relative) decides
// only when they differ by more than 2^-40; otherwise the 256-bit products do.
__device__ __forceinline__ bool better(const Cand &a, const Cand &b) {
    if (a.k == 0) return false;
    if (b.k == 0) return true;
    const double L = __dmul_rn(a.x, b.dp), R = __dmul_rn(b.x, a.dp);
    const double tol = 1.0 + 0x1p-40;
    if (L > __dmul_rn(R, tol)) return true;
    if (R > __dmul_rn(L, tol)) return false;
    const int c = exact_cmp(a, b);
    if (c != 0) return c > 0;
    return a.k < b.k;
}

// ---------------------------------------------------------------- sampled prefix moments
// PS1[j] = sum_{i < 32 j} t[i] (u64), PS2[j] = sum_{i < 32 j} t[i]^2 (u128).
// Prefix at any row x = chunk prefix + at most 31 loads of t.
constexpr int kChunkLog = 5;
constexpr uint64_t kChunk = 1ull << kChunkLog;

// The partial chunk [32 (x / 32), x) lies in one 128-byte line: read with up to
// eight independent uint4 loads (all in flight) when t is 16-byte aligned.
__device__ __forceinline__ uint64_t pref1(const uint64_t *PS1, const uint32_t *t, uint64_t x) {
    uint64_t s = PS1[x >> kChunkLog];
    const uint32_t r = (uint32_t)(x & (kChunk - 1));
    const uint64_t b = x - r;
    if (r && (reinterpret_cast<uintptr_t>(t) & 15) == 0) {
        const uint4 *c = reinterpret_cast<const uint4 *>(t + b);
#pragma unroll
        for (uint32_t k = 0; k < kChunk / 4; k++)
            if (4 * k < r) {
                const uint4 v = c[k];
                s += v.x + (4 * k + 1 < r ? (uint64_t)v.y : 0) + (4 * k + 2 < r ? (uint64_t)v.z : 0) +
                     (4 * k + 3 < r ? (uint64_t)v.w : 0);
            }
        return s;
    }
    for (uint64_t i = b; i < x; i++) s += t[i];
    return s;
}

__device__ __forceinline__ void pref12(const uint64_t *PS1, const u128 *PS2, const uint32_t *t, uint64_t x,
                                       uint64_t &s, u128 &q) {
    s = PS1[x >> kChunkLog];
    q = PS2[x >> kChunkLog];
    const uint32_t r = (uint32_t)(x & (kChunk - 1));
    const uint64_t b = x - r;
    if (r && (reinterpret_cast<uintptr_t>(t) & 15) == 0) {
        const uint4 *c = reinterpret_cast<const uint4 *>(t + b);
#pragma unroll
        for (uint32_t k = 0; k < kChunk / 4; k++)
            if (4 * k < r) {
                const uint4 v = c[k];
                const uint64_t e0 = v.x, e1 = 4 * k + 1 < r ? v.y : 0u, e2 = 4 * k + 2 < r ? v.z : 0u,
                               e3 = 4 * k + 3 < r ? v.w : 0u;
                s += e0 + e1 + e2 + e3;
                q += (u128)(e0 * e0) + (e1 * e1) + (u128)(e2 * e2) + (e3 * e3);
            }
        return;
    }
    for (uint64_t i = b; i < x; i++) {
        const uint64_t v = t[i];
        s += v;
        q += (u128)(v * v);
    }
}

// ---------------------------------------------------------------- Philox4x32-10
struct U4 { uint32_t x, y, z, w; };

__device__ __forceinline__ U4 philox4x32_10(U4 c, uint32_t k0, uint32_t k1) {
#pragma unroll
    for (int r = 0; r < 10; r++) {
        const uint32_t lo0 = 0xD2511F53u * c.x, hi0 = __umulhi(0xD2511F53u, c.x);
        const uint32_t lo1 = 0xCD9E8D57u * c.z, hi1 = __umulhi(0xCD9E8D57u, c.z);
        c = U4{hi1 ^ c.y ^ k0, lo1, hi0 ^ c.w ^ k1, lo0};
        k0 += 0x9E3779B9u;
        k1 += 0xBB67AE85u;
    }
    return c;
}

// ---------------------------------------------------------------- search
// number of elements of sorted a[0..n) that are <= x
template <class T>
__device__ __forceinline__ uint64_t upper_bound(const T *a, uint64_t n, T x) {
    uint64_t lo = 0, hi = n;
    while (lo < hi) {
        const uint64_t mid = (lo + hi) >> 1;
        if (a[mid] <= x) lo = mid + 1; else hi = mid;
    }
    return lo;
}

// number of elements of sorted a[0..n) that are < x
template <class T>
__device__ __forceinline__ uint64_t lower_bound(const T *a, uint64_t n, T x) {
    uint64_t lo = 0, hi = n;
    while (lo < hi) {
        const uint64_t mid = (lo + hi) >> 1;
        if (a[mid] < x) lo = mid + 1; else hi = mid;
    }
    return lo;
}

// ---------------------------------------------------------------- warp / block scans
template <class T>
__device__ __forceinline__ T shfl_up_t(T v, int d) {
    if constexpr (sizeof(T) <= 8) {
        return __shfl_up_sync(0xffffffffu, v, d);
    } else {
        static_assert(sizeof(T) % 8 == 0, "shuffle size");
        union { T v; uint64_t w[sizeof(T) / 8]; } u;
        u.v = v;
#pragma unroll
        for (int i = 0; i < (int)(sizeof(T) / 8); i++) u.w[i] = __shfl_up_sync(0xffffffffu, u.w[i], d);
        return u.v;
    }
}

// Inclusive warp scan with +.
template <class T>
__device__ __forceinline__ T warp_incl_scan(T v) {
    const int lane = threadIdx.x & 31;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
        T o = shfl_up_t(v, d);
        if (lane >= d) v = v + o;
    }
    return v;
}

// Exclusive block scan of one value per thread (+); returns exclusive prefix,
// writes block total to *total.  smem: NW entries of T.  All threads call.
template <class T, int NT>
__device__ __forceinline__ T block_excl_scan(T v, T *smem, T *total) {
    constexpr int NW = NT / 32;
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    const T incl = warp_incl_scan(v);
    if (lane == 31) smem[w] = incl;
    __syncthreads();
    if (w == 0) {
        T x = lane < NW ? smem[lane] : T{};
        T xi = warp_incl_scan(x);
        if (lane < NW) smem[lane] = xi - x;  // exclusive
        if (lane == NW - 1) smem[NW] = xi;
    }
    __syncthreads();
    const T r = smem[w] + (incl - v);
    *total = smem[NW];
    __syncthreads();
    return r;
}

}  // namespace sr
