// sort.cu -- step a1 (group by kernel): stable LSD radix sort of a
// compact (kernel_id, t) key carrying the trace row, one-sweep style (Adinets
// & Merrill): every pass reads and writes the data once; tiles get their
// global digit offsets by decoupled look-back.
//
// Offset key.  key = B[kid] + t, where B is the exclusive scan of
// W[k] = roundup(max_t[k] + 1, 2^16) over the kernels present (0 for absent
// ones).  Lexicographic (kid, t) order equals key order, and the key range is
// sum_k W[k] instead of K * 2^tbits: for C5 (10k kernels, lognormal tails up
// to 2^32 ns) ~2^38 instead of 2^46, so 5 byte passes instead of 6.  Because
// every B[k] is a multiple of 2^16, the low two key bytes are the low two
// bytes of t: the pre-pass (one read of the trace, before B is known) gives
// their histograms; the first pass histograms the higher key bytes as it
// reads the keys.  The last pass recovers kid from key >> 16 through a table
// (B[k] >> 16 .. B[k+1] >> 16 -> k), or by binary search over B when the
// table would be large, and writes t = key - B[kid].
//
// Coarse bases.  When rounding W[k] up to 2^24 instead costs no extra pass,
// B[k] is a multiple of 2^24: key byte 2 is t byte 2, and key bits 24.. are
// (B[k] >> 24) + (t >> 24), so every pass histogram comes from the pre-pass
// (t bytes 0-2, and a per-kernel histogram of t >> 24 that only the rare rows
// with t >= 2^24 touch) and the first pass does no extra counting.
//
// Packed mode (no payload).  When the key needs `bits` bits, the u64 holds
// (B[kid] + t) << s | (row mod 2^s), s = 64 - bits: the passes sort on the
// digits at s + 8p and the low row bits ride along for free, so every pass
// moves 8 B per row instead of 12.  Equal keys keep row order (stable LSD), so
// the last pass writes t and the low row bits in (kid, t, row) order; the
// sample stage recovers a full row from its low bits by checking the
// ceil(n / 2^s) candidate rows against the trace (stem.cu, R14 unchanged).
#include <cstdlib>

#include "internal.h"

namespace sr {

constexpr uint64_t kFlagA = 1ull << 62, kFlagP = 2ull << 62, kValMask = (1ull << 62) - 1;

// Look-back statuses are u32 (flag in bits 30-31, count in bits 0-29) when
// n < 2^30, else u64 (flag in bits 62-63): half the status traffic and clear.
__device__ __forceinline__ void put_status(uint64_t *st, bool s32, uint64_t idx, uint64_t flag, uint64_t val) {
    if (s32) __stcg(reinterpret_cast<uint32_t *>(st) + idx, (uint32_t)(flag >> 32) | (uint32_t)val);
    else __stcg(st + idx, flag | val);
}
__device__ __forceinline__ uint64_t get_status(const uint64_t *st, bool s32, uint64_t idx) {
    if (s32) {
        const uint32_t v = *(volatile const uint32_t *)(reinterpret_cast<const uint32_t *>(st) + idx);
        return ((uint64_t)(v >> 30) << 62) | (v & 0x3FFFFFFFu);
    }
    return *(volatile const uint64_t *)(st + idx);
}
constexpr int kMaxPasses = 8;
constexpr int kRB = 8, kR = 1 << kRB;       // byte digits
constexpr int kHistR = 256;                 // histogram row stride
constexpr int kBaseShift = 16;              // B[k] is a multiple of 2^16
constexpr uint64_t kMaxTable = 1ull << 27;  // kid-table entries (512 MB) before binary search
#ifndef SR_SORT_LB
#define SR_SORT_LB 4
#endif
#ifndef SR_SORT_LSMERGE
#define SR_SORT_LSMERGE 1
#endif
#ifndef SR_SORT_MINB
#define SR_SORT_MINB 4
#endif
constexpr int kLB = SR_SORT_LB;             // look-back: predecessor statuses read per round trip
constexpr int kCoarseShift = 24;            // coarse bases: B[k] a multiple of 2^24
constexpr uint32_t kMaxTailK = 1u << 16;    // coarse bases need a [K][256] tail histogram
constexpr int kHistT2 = kMaxPasses;         // hist row of t byte 2 (pre-pass)

// ---------------------------------------------------------------- pre-pass
// kernel-id counts (group sizes), per-kernel max t, kernel-id range check, max
// t, the histograms of t bytes 0 and 1 (= key bytes 0 and 1) and 2 (row
// kHistT2), and (tailh != NULL) the per-kernel histogram of t >> 24 >= 1.
constexpr int kPreThreads = 1024;
__global__ void __launch_bounds__(kPreThreads, 2) prepass_kernel(const uint32_t *__restrict__ kid, const uint32_t *__restrict__ t,
                                                      uint64_t n, uint32_t K, int smem_kid,
                                                      uint32_t *__restrict__ kid_count, uint32_t *__restrict__ kid_max,
                                                      uint64_t *__restrict__ hist, uint32_t *__restrict__ max_t,
                                                      uint32_t *__restrict__ err, uint32_t *__restrict__ tailh,
                                                      int nc) {
    // [nc][3][256] byte histograms (copy = lane mod nc, stride 3*256+1 words so
    // a bin's copies sit in different banks: equal bytes within a warp collide
    // on one address nc times less often), then [K] counts, [K] max
    extern __shared__ uint32_t sh[];
    constexpr int HS = 3 * kR + 1;
    uint32_t *hk = sh + nc * HS, *hm = hk + (smem_kid ? K : 0);
    uint32_t *h0 = sh + (threadIdx.x & (nc - 1)) * HS;
    for (int i = threadIdx.x; i < nc * HS; i += blockDim.x) sh[i] = 0;
    if (smem_kid)
        for (uint32_t i = threadIdx.x; i < 2 * K; i += blockDim.x) hk[i] = 0;
    __syncthreads();
    uint32_t mx = 0, bad = 0;
    const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    const uint64_t n4 = n / 4;
    const uint4 *kid4 = reinterpret_cast<const uint4 *>(kid), *t4 = reinterpret_cast<const uint4 *>(t);
    auto one = [&](uint32_t k, uint32_t x) {
        mx = max(mx, x);
        atomicAdd(&h0[x & (kR - 1)], 1u);
        atomicAdd(&h0[kR + ((x >> kRB) & (kR - 1))], 1u);
        if ((x >> (2 * kRB)) & (kR - 1)) atomicAdd(&h0[2 * kR + ((x >> (2 * kRB)) & (kR - 1))], 1u);   // bin 0: n - rest
        if (k >= K) { bad = 1; return; }
        if (tailh && (x >> kCoarseShift)) atomicAdd(&tailh[(uint64_t)k * kR + (x >> kCoarseShift)], 1u);
        if (smem_kid) {
            atomicAdd(&hk[k], 1u);
            if (x > hm[k]) atomicMax(&hm[k], x);   // a read first: most rows do not raise the max
        } else {
            atomicAdd(&kid_count[k], 1u);
            atomicMax(&kid_max[k], x);
        }
    };
    const bool aligned = ((reinterpret_cast<uintptr_t>(kid) | reinterpret_cast<uintptr_t>(t)) & 15) == 0;
    if (aligned) {
        uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
        for (; i + stride < n4; i += 2 * stride) {   // two uint4 pairs in flight per thread
            const uint4 a = __ldg(kid4 + i), b = __ldg(t4 + i);
            const uint4 a2 = __ldg(kid4 + i + stride), b2 = __ldg(t4 + i + stride);
            one(a.x, b.x); one(a.y, b.y); one(a.z, b.z); one(a.w, b.w);
            one(a2.x, b2.x); one(a2.y, b2.y); one(a2.z, b2.z); one(a2.w, b2.w);
        }
        for (; i < n4; i += stride) {
            const uint4 a = __ldg(kid4 + i), b = __ldg(t4 + i);
            one(a.x, b.x); one(a.y, b.y); one(a.z, b.z); one(a.w, b.w);
        }
        for (uint64_t i = n4 * 4 + (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += stride)
            one(__ldg(kid + i), __ldg(t + i));
    } else {
        for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += stride)
            one(__ldg(kid + i), __ldg(t + i));
    }
    for (int o = 16; o; o >>= 1) {
        mx = max(mx, __shfl_xor_sync(0xffffffffu, mx, o));
        bad |= __shfl_xor_sync(0xffffffffu, bad, o);
    }
    if ((threadIdx.x & 31) == 0) {
        if (mx) atomicMax(max_t, mx);
        if (bad) atomicOr(err, 1u);
    }
    __syncthreads();
    for (int i = threadIdx.x; i < 3 * kR; i += blockDim.x) {
        uint32_t v = 0;
        for (int cp = 0; cp < nc; cp++) v += sh[cp * HS + i];
        if (v) atomicAdd((unsigned long long *)&hist[((i >> kRB) == 2 ? kHistT2 : (i >> kRB)) * kHistR + (i & (kR - 1))],
                         (unsigned long long)v);
    }
    if (smem_kid)
        for (uint32_t i = threadIdx.x; i < K; i += blockDim.x)
            if (hk[i]) {
                atomicAdd(&kid_count[i], hk[i]);
                atomicMax(&kid_max[i], hm[i]);
            }
}

// The pre-pass over whole 5 120-row sort tiles (the first pass's tile shape):
// besides everything prepass_kernel counts, each tile's histogram of t byte 0
// (the first pass's digit) goes to tileh[tile][256] (u16).  Their column
// prefix sums give every first-pass tile its global digit offsets, so the
// first pass needs no decoupled look-back (tile_excl_*_kernel below).
#ifndef SR_PRET_THREADS
#define SR_PRET_THREADS 1024
#endif
#ifndef SR_PRET_MINB
#define SR_PRET_MINB 2
#endif
#ifndef SR_PRET_PAIRS
#define SR_PRET_PAIRS 1
#endif
constexpr int kPreTThreads = SR_PRET_THREADS;              // kPreTiles tiles per step = five uint4 per thread
constexpr int kPreTiles = kPreTThreads * 5 * 4 / 5120;     // 512 threads: 2 tiles, 1024: 4
__global__ void __launch_bounds__(kPreTThreads, SR_PRET_MINB) prepass_tile_kernel(
    const uint32_t *__restrict__ kid, const uint32_t *__restrict__ t, uint64_t n, uint32_t K, int smem_kid,
    uint32_t *__restrict__ kid_count, uint32_t *__restrict__ kid_max, uint64_t *__restrict__ hist,
    uint32_t *__restrict__ max_t, uint32_t *__restrict__ err, uint32_t *__restrict__ tailh,
    uint16_t *__restrict__ tileh, uint64_t tile0, uint32_t tile_rows) {
    extern __shared__ uint32_t sh[];
    // [3][256] block histograms of t bytes 0..2 (byte 0 from the tile histograms),
    // [kPreTiles][256] the current tiles', [K] counts, [K] max
    uint32_t *h0 = sh, *th = sh + 3 * kR, *hk = th + kPreTiles * kR, *hm = hk + (smem_kid ? K : 0);
    for (int i = threadIdx.x; i < (3 + kPreTiles) * kR; i += blockDim.x) sh[i] = 0;
    if (smem_kid)
        for (uint32_t i = threadIdx.x; i < 2 * K; i += blockDim.x) hk[i] = 0;
    __syncthreads();
    uint32_t mx = 0, bad = 0;
    auto one = [&](uint32_t *tq, uint32_t k, uint32_t x) {
        mx = max(mx, x);
        atomicAdd(&tq[x & (kR - 1)], 1u);
        atomicAdd(&h0[kR + ((x >> kRB) & (kR - 1))], 1u);
        if ((x >> (2 * kRB)) & (kR - 1)) atomicAdd(&h0[2 * kR + ((x >> (2 * kRB)) & (kR - 1))], 1u);
        if (k >= K) { bad = 1; return; }
        if (tailh && (x >> kCoarseShift)) atomicAdd(&tailh[(uint64_t)k * kR + (x >> kCoarseShift)], 1u);
        if (smem_kid) {
            atomicAdd(&hk[k], 1u);
            if (x > hm[k]) atomicMax(&hm[k], x);
        } else {
            atomicAdd(&kid_count[k], 1u);
            atomicMax(&kid_max[k], x);
        }
    };
    const uint64_t ntiles = (n + tile_rows - 1) / tile_rows, nsteps = (ntiles + kPreTiles - 1) / kPreTiles;
    const uint4 *kid4 = reinterpret_cast<const uint4 *>(kid), *t4 = reinterpret_cast<const uint4 *>(t);
    const bool aligned = ((reinterpret_cast<uintptr_t>(kid) | reinterpret_cast<uintptr_t>(t)) & 15) == 0 &&
                         tile_rows % 4 == 0;
    const uint32_t q4 = tile_rows / 4;   // uint4 per tile
    for (uint64_t sidx = blockIdx.x; sidx < nsteps; sidx += gridDim.x) {
        const uint64_t q0 = sidx * kPreTiles, r0 = q0 * tile_rows;
        const uint64_t cnt = min((uint64_t)kPreTiles * tile_rows, n - r0);
        if (aligned && cnt == (uint64_t)kPreTiles * tile_rows && kPreTiles * q4 == 5 * kPreTThreads) {
#if SR_PRET_PAIRS == 5
            uint4 a[5], b[5];
#pragma unroll
            for (int k = 0; k < 5; k++) {
                a[k] = __ldg(kid4 + r0 / 4 + threadIdx.x + k * kPreTThreads);
                b[k] = __ldg(t4 + r0 / 4 + threadIdx.x + k * kPreTThreads);
            }
#pragma unroll
            for (int k = 0; k < 5; k++) {
                uint32_t *tq = th + ((threadIdx.x + k * kPreTThreads) / q4) * kR;
                one(tq, a[k].x, b[k].x); one(tq, a[k].y, b[k].y); one(tq, a[k].z, b[k].z); one(tq, a[k].w, b[k].w);
            }
#else   // SR_PRET_PAIRS uint4 pairs in flight per thread (fewer registers: more warps per SM)
#pragma unroll 1
            for (int k0 = 0; k0 < 5; k0 += SR_PRET_PAIRS) {
                uint4 a[SR_PRET_PAIRS], b[SR_PRET_PAIRS];
#pragma unroll
                for (int k = 0; k < SR_PRET_PAIRS; k++)
                    if (k0 + k < 5) {
                        a[k] = __ldg(kid4 + r0 / 4 + threadIdx.x + (k0 + k) * kPreTThreads);
                        b[k] = __ldg(t4 + r0 / 4 + threadIdx.x + (k0 + k) * kPreTThreads);
                    }
#pragma unroll
                for (int k = 0; k < SR_PRET_PAIRS; k++)
                    if (k0 + k < 5) {
                        uint32_t *tq = th + ((threadIdx.x + (k0 + k) * kPreTThreads) / q4) * kR;
                        one(tq, a[k].x, b[k].x); one(tq, a[k].y, b[k].y); one(tq, a[k].z, b[k].z);
                        one(tq, a[k].w, b[k].w);
                    }
            }
#endif
        } else {
            for (uint64_t i = threadIdx.x; i < cnt; i += blockDim.x)
                one(th + (i / tile_rows) * kR, __ldg(kid + r0 + i), __ldg(t + r0 + i));
        }
        __syncthreads();
        for (int i = threadIdx.x; i < kPreTiles * kR; i += blockDim.x) {
            const uint64_t q = q0 + (i >> kRB);
            const uint32_t v = th[i];
            if (q < ntiles) {
                tileh[(tile0 + q) * kR + (i & (kR - 1))] = (uint16_t)v;
                atomicAdd(&h0[i & (kR - 1)], v);
            }
            th[i] = 0;
        }
        __syncthreads();
    }
    for (int o = 16; o; o >>= 1) {
        mx = max(mx, __shfl_xor_sync(0xffffffffu, mx, o));
        bad |= __shfl_xor_sync(0xffffffffu, bad, o);
    }
    if ((threadIdx.x & 31) == 0) {
        if (mx) atomicMax(max_t, mx);
        if (bad) atomicOr(err, 1u);
    }
    __syncthreads();
    for (int i = threadIdx.x; i < 3 * kR; i += blockDim.x) {
        const uint32_t v = sh[i];
        if (v) atomicAdd((unsigned long long *)&hist[((i >> kRB) == 2 ? kHistT2 : (i >> kRB)) * kHistR + (i & (kR - 1))],
                         (unsigned long long)v);
    }
    if (smem_kid)
        for (uint32_t i = threadIdx.x; i < K; i += blockDim.x)
            if (hk[i]) {
                atomicAdd(&kid_count[i], hk[i]);
                atomicMax(&kid_max[i], hm[i]);
            }
}

// The same pre-pass with the tiles dealt to WARPS: each warp keeps its tile's
// digit histogram in shared memory (two u16 counts per word), so no block
// barrier is needed between tiles and warps drift as in prepass_kernel.
__global__ void __launch_bounds__(1024, 2) prepass_wtile_kernel(
    const uint32_t *__restrict__ kid, const uint32_t *__restrict__ t, uint64_t n, uint32_t K, int smem_kid,
    uint32_t *__restrict__ kid_count, uint32_t *__restrict__ kid_max, uint64_t *__restrict__ hist,
    uint32_t *__restrict__ max_t, uint32_t *__restrict__ err, uint32_t *__restrict__ tailh,
    uint16_t *__restrict__ tileh, uint64_t tile0, uint32_t tile_rows) {
    extern __shared__ uint32_t sh[];
    // [3][256] block histograms of t bytes 0..2, [32 warps][128] packed tile counts, [K] counts, [K] max
    constexpr int NW = 1024 / 32, TW = kR / 2;
    uint32_t *h0 = sh, *tw = sh + 3 * kR, *hk = tw + NW * TW, *hm = hk + (smem_kid ? K : 0);
    for (int i = threadIdx.x; i < 3 * kR + NW * TW; i += blockDim.x) sh[i] = 0;
    if (smem_kid)
        for (uint32_t i = threadIdx.x; i < 2 * K; i += blockDim.x) hk[i] = 0;
    __syncthreads();
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    uint32_t *th = tw + w * TW;
    uint32_t mx = 0, bad = 0;
    auto one = [&](uint32_t k, uint32_t x) {
        mx = max(mx, x);
        atomicAdd(&th[(x & (kR - 1)) >> 1], 1u << (16 * (x & 1)));
        atomicAdd(&h0[kR + ((x >> kRB) & (kR - 1))], 1u);
        if ((x >> (2 * kRB)) & (kR - 1)) atomicAdd(&h0[2 * kR + ((x >> (2 * kRB)) & (kR - 1))], 1u);
        if (k >= K) { bad = 1; return; }
        if (tailh && (x >> kCoarseShift)) atomicAdd(&tailh[(uint64_t)k * kR + (x >> kCoarseShift)], 1u);
        if (smem_kid) {
            atomicAdd(&hk[k], 1u);
            if (x > hm[k]) atomicMax(&hm[k], x);
        } else {
            atomicAdd(&kid_count[k], 1u);
            atomicMax(&kid_max[k], x);
        }
    };
    const uint64_t ntiles = (n + tile_rows - 1) / tile_rows;
    const uint64_t gw = (uint64_t)blockIdx.x * NW + w, nwarps = (uint64_t)gridDim.x * NW;
    const uint4 *kid4 = reinterpret_cast<const uint4 *>(kid), *t4 = reinterpret_cast<const uint4 *>(t);
    const bool aligned = ((reinterpret_cast<uintptr_t>(kid) | reinterpret_cast<uintptr_t>(t)) & 15) == 0 &&
                         tile_rows % 128 == 0;
    for (uint64_t q = gw; q < ntiles; q += nwarps) {
        const uint64_t r0 = q * tile_rows, cnt = min((uint64_t)tile_rows, n - r0);
        if (aligned && cnt == tile_rows) {
            const uint64_t j0 = r0 / 4;
            const uint32_t nj = tile_rows / 4;
#pragma unroll 2
            for (uint32_t j = lane; j < nj; j += 32) {
                const uint4 a = __ldg(kid4 + j0 + j), b = __ldg(t4 + j0 + j);
                one(a.x, b.x); one(a.y, b.y); one(a.z, b.z); one(a.w, b.w);
            }
        } else {
            for (uint64_t i = lane; i < cnt; i += 32) one(__ldg(kid + r0 + i), __ldg(t + r0 + i));
        }
        __syncwarp();
#pragma unroll
        for (int u = 0; u < TW / 32; u++) {   // 4 words (8 digits) per lane: out, into the block's byte-0 counts, zero
            const int wi = lane + 32 * u;
            const uint32_t v = th[wi];
            th[wi] = 0;
            reinterpret_cast<uint32_t *>(tileh + (tile0 + q) * kR)[wi] = v;   // the two u16 counts, in place
            if (v & 0xFFFFu) atomicAdd(&h0[2 * wi], v & 0xFFFFu);
            if (v >> 16) atomicAdd(&h0[2 * wi + 1], v >> 16);
        }
        __syncwarp();
    }
    for (int o = 16; o; o >>= 1) {
        mx = max(mx, __shfl_xor_sync(0xffffffffu, mx, o));
        bad |= __shfl_xor_sync(0xffffffffu, bad, o);
    }
    if (lane == 0) {
        if (mx) atomicMax(max_t, mx);
        if (bad) atomicOr(err, 1u);
    }
    __syncthreads();
    for (int i = threadIdx.x; i < 3 * kR; i += blockDim.x) {
        const uint32_t v = sh[i];
        if (v) atomicAdd((unsigned long long *)&hist[((i >> kRB) == 2 ? kHistT2 : (i >> kRB)) * kHistR + (i & (kR - 1))],
                         (unsigned long long)v);
    }
    if (smem_kid)
        for (uint32_t i = threadIdx.x; i < K; i += blockDim.x)
            if (hk[i]) {
                atomicAdd(&kid_count[i], hk[i]);
                atomicMax(&kid_max[i], hm[i]);
            }
}

// Global first-pass offsets per tile from the tile histograms: excl[q][d] =
// the rows of digit d in tiles before q.  Groups of kExGrp tiles: their
// column sums, a scan of those per digit, then the tiles of each group.
constexpr int kExGrp = 64;
__global__ void tile_grp_kernel(const uint16_t *__restrict__ tileh, uint64_t ntiles, uint32_t *__restrict__ grp) {
    const uint64_t g = blockIdx.x, q0 = g * kExGrp, q1 = min(q0 + kExGrp, ntiles);
    uint32_t s = 0;
#pragma unroll 16
    for (uint64_t q = q0; q < q1; q++) s += tileh[q * kR + threadIdx.x];
    grp[g * kR + threadIdx.x] = s;
}
// one block per digit: exclusive scan of its column of group sums (in place)
__global__ void __launch_bounds__(1024) grp_scan_kernel(uint32_t *__restrict__ grp, uint64_t ngrp) {
    __shared__ uint32_t s_w[32];
    const uint32_t d = blockIdx.x;
    uint32_t carry = 0;
    for (uint64_t b0 = 0; b0 < ngrp; b0 += 1024) {
        const uint64_t g = b0 + threadIdx.x;
        const uint32_t v = g < ngrp ? grp[g * kR + d] : 0u;
        uint32_t incl = v;
        const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
        for (int o = 1; o < 32; o <<= 1) {
            const uint32_t u = __shfl_up_sync(0xffffffffu, incl, o);
            if (lane >= o) incl += u;
        }
        if (lane == 31) s_w[w] = incl;
        __syncthreads();
        uint32_t off = 0;
        for (int k = 0; k < w; k++) off += s_w[k];
        uint32_t tot = 0;
        for (int k = 0; k < 32; k++) tot += s_w[k];
        if (g < ngrp) grp[g * kR + d] = carry + off + incl - v;
        carry += tot;
        __syncthreads();
    }
}
__global__ void tile_excl_kernel(const uint16_t *__restrict__ tileh, uint64_t ntiles, const uint32_t *__restrict__ grp,
                                 uint32_t *__restrict__ excl) {
    const uint64_t g = blockIdx.x, q0 = g * kExGrp;
    uint32_t run = grp[g * kR + threadIdx.x];
    for (int h = 0; h < kExGrp; h += 16) {   // 16 loads in flight, then the running sums
        uint32_t v[16];
#pragma unroll
        for (int u = 0; u < 16; u++) {
            const uint64_t q = q0 + h + u;
            v[u] = q < ntiles ? tileh[q * kR + threadIdx.x] : 0u;
        }
#pragma unroll
        for (int u = 0; u < 16; u++) {
            const uint64_t q = q0 + h + u;
            if (q < ntiles) excl[q * kR + threadIdx.x] = run;
            run += v[u];
        }
    }
}

// kid-table entry j -> the kernel whose key range holds j << tsh
__global__ void kid_table_kernel(const uint64_t *__restrict__ B, uint32_t K, uint64_t entries, int tsh,
                                 uint32_t *__restrict__ tab) {
    const uint64_t j = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (j >= entries) return;
    tab[j] = (uint32_t)(upper_bound(B, (uint64_t)K + 1, j << tsh) - 1);
}

__global__ void base_shift_kernel(const uint64_t *__restrict__ B, uint64_t m, int tsh, uint32_t *__restrict__ Bs,
                                  uint16_t *__restrict__ Bs16) {
    const uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= m) return;
    if (Bs16) Bs16[i] = (uint16_t)(B[i] >> tsh);
    else Bs[i] = (uint32_t)(B[i] >> tsh);
}

// Coarse bases: histograms of key bytes 2 .. npasses-1 from the pre-pass.
// Byte 2 is t byte 2; bits 24.. of kernel k's keys are (B[k] >> 24) + u for
// its rows with t >> 24 = u.  One warp per kernel.
__global__ void coarse_hist_kernel(const uint32_t *__restrict__ cnt, const uint32_t *__restrict__ tailh,
                                   const uint64_t *__restrict__ B, uint32_t K, int npasses, uint64_t n,
                                   uint64_t *__restrict__ hist) {
    if (blockIdx.x == 0 && npasses > 2) {   // t byte 2; the pre-pass counts bins >= 1 only
        __shared__ uint64_t s_part[8];
        const uint64_t h = threadIdx.x ? hist[kHistT2 * kHistR + threadIdx.x] : 0;
        uint64_t v = h;
        for (int o = 16; o; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
        if ((threadIdx.x & 31) == 0) s_part[threadIdx.x >> 5] = v;
        __syncthreads();
        uint64_t rest = 0;
        for (int w = 0; w < 8; w++) rest += s_part[w];
        hist[2 * kHistR + threadIdx.x] = threadIdx.x ? h : n - rest;
    }
    const uint32_t k = blockIdx.x * (blockDim.x / 32) + (threadIdx.x >> 5), lane = threadIdx.x & 31;
    if (k >= K || cnt[k] == 0) return;
    const uint64_t v0 = B[k] >> kCoarseShift;
    auto add = [&](uint64_t v, uint32_t c) {
        for (int x = 3; x < npasses; x++)
            atomicAdd((unsigned long long *)&hist[x * kHistR + ((v >> (kRB * (x - 3))) & (kR - 1))],
                      (unsigned long long)c);
    };
    uint32_t tail = 0;
    for (uint32_t u = 1 + lane; u < (uint32_t)kR; u += 32) {
        const uint32_t c = tailh[(uint64_t)k * kR + u];
        if (c) { tail += c; add(v0 + u, c); }
    }
    for (int o = 16; o; o >>= 1) tail += __shfl_xor_sync(0xffffffffu, tail, o);
    if (lane == 0) add(v0, cnt[k] - tail);
}

// Per pass, from its digit histogram: the digit bases (exclusive scan) and
// the ranking mode.  MATCH.ANY slows down as the number of distinct digits
// among a warp's 32 keys approaches 32, while 8 ballots cost the same for any
// digit mix.  Measured on B200 (C5, 5 passes; whole sort ms all-ballot /
// all-match: first 6.8/9.4, mid 16.1/18.9, last 5.8/5.3; threshold 16/20/24:
// last pass 5.09/5.09/4.76): ballots when E[distinct] >= 24.  force >= 0
// fixes the mode.
__global__ void rank_mode_kernel(const uint64_t *__restrict__ hist, int p0, int p1, uint64_t n, int force,
                                 double thr, uint32_t *__restrict__ mode, uint64_t *__restrict__ gbase) {
    __shared__ double s_w[8];
    __shared__ uint64_t s_c[8];
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    for (int p = p0; p < p1; p++) {
        const uint64_t h = hist[p * kHistR + threadIdx.x];
        const double q = (double)h / (double)n;
        double e = 1.0 - pow(1.0 - q, 32.0);
        for (int o = 16; o; o >>= 1) e += __shfl_xor_sync(0xffffffffu, e, o);
        uint64_t inc = h;
        for (int o = 1; o < 32; o <<= 1) {
            const uint64_t v = __shfl_up_sync(0xffffffffu, inc, o);
            if (lane >= o) inc += v;
        }
        if (lane == 0) s_w[w] = e;
        if (lane == 31) s_c[w] = inc;
        __syncthreads();
        uint64_t off = 0;
        for (int k = 0; k < w; k++) off += s_c[k];
        gbase[p * kHistR + threadIdx.x] = off + inc - h;
        if (threadIdx.x == 0) {
            double tot = 0.0;
            for (int i = 0; i < 8; i++) tot += s_w[i];
            mode[p] = force >= 0 ? (uint32_t)force : tot >= thr ? 1u : 0u;
        }
        __syncthreads();
    }
}

// Lanes of vmask whose 8-bit digit differs from this lane's d: one ballot per
// bit, mismatches = ballot ^ (my bit ? ~0 : 0), OR-accumulated (4 SASS per bit).
__device__ __forceinline__ uint32_t ballot_diff8(uint32_t d, uint32_t vmask) {
    uint32_t diff;
    asm("{\n\t.reg .pred p;\n\t.reg .b32 b, m, acc;\n\t"
        "mov.b32 acc, 0;\n\t"
#define SR_BAL_BIT(K) "and.b32 m, %1, " #K ";\n\tsetp.ne.u32 p, m, 0;\n\tvote.sync.ballot.b32 b, p, %2;\n\t" \
                      "selp.b32 m, -1, 0, p;\n\txor.b32 b, b, m;\n\tor.b32 acc, acc, b;\n\t"
        SR_BAL_BIT(1) SR_BAL_BIT(2) SR_BAL_BIT(4) SR_BAL_BIT(8) SR_BAL_BIT(16) SR_BAL_BIT(32) SR_BAL_BIT(64)
        SR_BAL_BIT(128)
#undef SR_BAL_BIT
        "mov.b32 %0, acc;\n\t}"
        : "=r"(diff)
        : "r"(d), "r"(vmask));
    return diff;
}

// ---------------------------------------------------------------- one-sweep pass
// a streaming 4-byte load that does not allocate in L1
__device__ __forceinline__ uint32_t ld_na(const uint32_t *p) {
    uint32_t v;
    asm("ld.global.nc.L1::no_allocate.b32 %0, [%1];" : "=r"(v) : "l"(p));   // read-only for the kernel
    return v;
}

struct PassArgs {
    const uint32_t *kid_in, *t_in;      // FIRST: trace columns
    const uint32_t *row_in;             // FIRST: row payload (NULL = the row index)
    const uint64_t *keys_in;            // !FIRST
    const uint32_t *vals_in;            // !FIRST
    uint64_t *keys_out;                 // !LAST
    uint32_t *vals_out;                 // !LAST
    uint32_t *t_out, *row_out;          // LAST
    const uint64_t *B;                  // [K + 1] key base per kernel
    const uint32_t *Bs;                 // [K + 1] B >> tsh (FIRST: a 4-byte gather that stays in L1)
    const uint16_t *Bs16;               // [K + 1] B >> tsh when it fits 16 bits (a 2-byte gather: half the L1 room)
    const uint32_t *tab;                // LAST: kid table (NULL: binary search over B)
    int tsh;                            // B[k] is a multiple of 2^tsh; LAST: kid-table index = key >> tsh
    uint64_t n;
    uint64_t lomask;                    // packed: low row bits kept in the key (2^ks - 1, <= 2^32 - 1)
    int ks;                             // packed: key shift s (0 in payload mode)
    uint32_t K;
    int shift, pass;
    int nxh;                            // FIRST: key bytes 2 .. 2 + nxh - 1 histogrammed here
    uint32_t pf;                        // tiles ahead to prefetch into L2 (0 = off)
    int late;                           // 1: publish the tile's digit counts after ranking
    int noalloc;                        // FIRST: stream kid / t past L1 (keeps the B[kid] table resident)
    uint32_t nap;                       // look-back: ns to sleep before re-polling an unpublished status
    const uint32_t *ballot;             // [pass] 1: equal-digit lanes by 8 ballots, 0: match.any
    const uint64_t *gbase;              // [pass][kHistR] exclusive scan of the pass's digit counts
    uint64_t *hist;                     // [pass][kHistR] global digit counts
    uint64_t *status;                   // [ntiles][R] (u32 words when s32)
    bool s32;                           // n < 2^30: 32-bit look-back statuses
    uint32_t *tile_counter;
    const uint32_t *tile_excl;          // FIRST: [tile][R] global offsets from the pre-pass (no look-back), or NULL
    uint64_t tile_base;                 // tile index of blockIdx.x 0 (with tile_excl)
};

// One LSD pass over digit (key >> shift) & 255.  NT threads, IT keys per
// thread; keys loaded warp-striped (coalesced), the tile's digit counts are
// published first (flag A), keys ranked in element order by warp-level
// multi-split (match.any), global offsets found by decoupled look-back
// (thread d < 256 owns digit d), then keys are staged in shared memory in
// tile-sorted order and written out in digit runs (coalesced).
template <int NT, int IT, bool FIRST, bool LAST, bool FULL, bool PK, bool S32>
__global__ void __launch_bounds__(NT, FULL ? (NT >= 448 ? 2 : NT >= 320 ? 3 : SR_SORT_MINB) : 1) onesweep_kernel(PassArgs a) {   // (FULL = false: one ragged tile; a looser bound avoids a ptxas C7600 failure)
    constexpr int NW = NT / 32, TILE = NT * IT, R = kR;
    static_assert(NT >= R, "one thread per digit");
    static_assert(NT * IT <= 65536, "16-bit ranks");
    extern __shared__ __align__(16) unsigned char s_dyn[];
    uint64_t *s_keys = reinterpret_cast<uint64_t *>(s_dyn);                           // [TILE]
    uint32_t *s_vals = reinterpret_cast<uint32_t *>(s_keys + TILE);                   // [TILE] (!PK)
    uint16_t (*s_whist)[R] = reinterpret_cast<uint16_t (*)[R]>(PK ? (void *)(s_keys + TILE) : (void *)(s_vals + TILE));
    __shared__ uint32_t s_delta[R];   // global - local position, mod 2^32 (n < 2^32)
    __shared__ uint32_t s_lstart[R + 1];
    __shared__ uint32_t s_cnt[R];
    __shared__ uint32_t s_cw[NW];
    __shared__ uint32_t s_tile;
    // FIRST: the extra digit histograms (a.nxh x R; dynamic, none with coarse bases)
    uint32_t *s_xh = reinterpret_cast<uint32_t *>(&s_whist[0][0] + NW * R);

    const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
    const bool nolb = FIRST && a.tile_excl;   // offsets known in advance: no look-back
    if (tid == 0) s_tile = nolb ? (uint32_t)(a.tile_base + blockIdx.x) : atomicAdd(a.tile_counter, 1u);
    for (int i = tid; i < NW * R / 2; i += NT) reinterpret_cast<uint32_t *>(&s_whist[0][0])[i] = 0;
    for (int i = tid; i < R; i += NT) s_cnt[i] = 0;
    if (FIRST)
        for (int i = tid; i < a.nxh * R; i += NT) s_xh[i] = 0;
    __syncthreads();
    const uint32_t tile = s_tile;
    const uint64_t wbase = (uint64_t)tile * TILE + (uint64_t)w * (32 * IT);
    // L2 prefetch of the tile that will be claimed pf tiles from now: its DRAM
    // reads overlap this tile's ranking and look-back (tiles are claimed in order)
    if (a.pf && tid < 2) {
        const uint64_t pt = (uint64_t)tile + a.pf, p0 = pt * TILE;
        if (p0 < a.n) {
            const uint64_t cnt = min((uint64_t)TILE, a.n - p0);
            const void *src;
            uint32_t bytes;
            if (FIRST) {
                src = tid == 0 ? (const void *)(a.kid_in + p0) : (const void *)(a.t_in + p0);
                bytes = (uint32_t)(cnt * 4);
            } else if (PK) {
                src = (const void *)(a.keys_in + p0 + (tid ? cnt / 2 : 0));
                bytes = (uint32_t)(tid ? (cnt - cnt / 2) * 8 : (cnt / 2) * 8);
            } else {
                src = tid == 0 ? (const void *)(a.keys_in + p0) : (const void *)(a.vals_in + p0);
                bytes = (uint32_t)(cnt * (tid == 0 ? 8 : 4));
            }
            bytes &= ~15u;
            if (bytes && (reinterpret_cast<uintptr_t>(src) & 15) == 0)
                asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(src), "r"(bytes) : "memory");
        }
    }

    uint64_t key[IT];
    uint32_t val[PK ? 1 : IT];
    if (FIRST && PK && a.Bs16 && a.noalloc) {
        // the common first pass (packed keys, 16-bit key-base table) as straight-line code
        const uint32_t lm = (uint32_t)a.lomask;
#pragma unroll
        for (int j = 0; j < IT; j++) {
            const uint64_t i = wbase + (uint64_t)j * 32 + lane;
            key[j] = ~0ull;
            if (FULL || i < a.n) {
                const uint32_t kd = ld_na(a.kid_in + i), tv = ld_na(a.t_in + i);
                const uint64_t kk = ((uint64_t)__ldg(a.Bs16 + kd) << a.tsh) + tv;
                key[j] = (kk << a.ks) | ((uint32_t)i & lm);
            }
        }
    } else
#pragma unroll
    for (int j = 0; j < IT; j++) {
        const uint64_t i = wbase + (uint64_t)j * 32 + lane;
        if (FULL || i < a.n) {
            if (FIRST) {
                const uint32_t kd = a.noalloc ? ld_na(a.kid_in + i) : __ldg(a.kid_in + i);
                const uint64_t kb = a.Bs16 ? (uint64_t)__ldg(a.Bs16 + kd) << a.tsh
                                    : a.Bs ? (uint64_t)__ldg(a.Bs + kd) << a.tsh : __ldg(a.B + kd);
                const uint64_t kk = kb + (uint64_t)(a.noalloc ? ld_na(a.t_in + i) : __ldg(a.t_in + i));
                if (PK) {
                    key[j] = (kk << a.ks) | (i & a.lomask);
                } else {
                    key[j] = kk;
                    val[PK ? 0 : j] = a.row_in ? __ldg(a.row_in + i) : (uint32_t)i;
                }
            } else {
                key[j] = __ldcs(a.keys_in + i);
                if (!PK) val[PK ? 0 : j] = __ldcs(a.vals_in + i);
            }
        } else {
            key[j] = ~0ull;
            if (!PK) val[PK ? 0 : j] = 0;
        }
    }
    // the tile's digit counts: either counted and published here, before
    // ranking (successors' look-backs need not wait for it), or (a.late, the
    // default: fewer instructions per key, measured faster) taken from the
    // ranking's warp histograms and published after ranking
    if (!a.late || (FIRST && a.nxh)) {
#pragma unroll
        for (int j = 0; j < IT; j++)
            if (FULL || wbase + (uint64_t)j * 32 + lane < a.n) {
                if (!a.late) atomicAdd(&s_cnt[(uint32_t)(key[j] >> a.shift) & (R - 1)], 1u);
                if (FIRST)
                    for (int x = 0; x < a.nxh; x++)
                        atomicAdd(&s_xh[x * R + ((uint32_t)(key[j] >> (a.ks + kBaseShift + kRB * x)) & (R - 1))], 1u);
            }
    }
    __syncthreads();
    if (tid < R && !a.late && !nolb) put_status(a.status, S32, (uint64_t)tile * R + tid, tile == 0 ? kFlagP : kFlagA, s_cnt[tid]);
    if (FIRST && tid < R)
        for (int x = 0; x < a.nxh; x++)
            if (s_xh[x * R + tid])
                atomicAdd((unsigned long long *)&a.hist[(2 + x) * kHistR + tid], (unsigned long long)s_xh[x * R + tid]);

    // warp-level multi-split ranking, in element order
    const uint32_t ballot = a.ballot[a.pass];
    uint32_t rank2[(IT + 1) / 2];   // two 16-bit ranks per register (ranks < TILE <= 2^16)
#pragma unroll
    for (int j = 0; j < IT; j++) {
        const uint64_t i = wbase + (uint64_t)j * 32 + lane;
        const bool valid = FULL || i < a.n;
        const uint32_t vmask = FULL ? 0xffffffffu : __ballot_sync(0xffffffffu, valid);
        if (valid) {
            const uint32_t d = (uint32_t)(key[j] >> a.shift) & (R - 1);
            uint32_t peers;
#ifdef SR_SORT_FAKE_RANK   // timing experiment only: no multi-split (wrong ranks)
            if (true) {
                peers = 1u << lane;
#else
            if (ballot) {
                peers = vmask & ~ballot_diff8(d, vmask);
#endif
            } else {
                peers = __match_any_sync(vmask, d);
            }
            const uint32_t base = s_whist[w][d];
            const uint32_t below = __popc(peers & ((1u << lane) - 1));
            if (j & 1) rank2[j / 2] |= (base + below) << 16;
            else rank2[j / 2] = base + below;
            __syncwarp(vmask);
            if (below == 0) s_whist[w][d] = (uint16_t)(base + __popc(peers));
        }
        __syncwarp();
    }
    __syncthreads();

    // local digit offsets (threads d < R): per-warp bases, tile-wide exclusive scan
    const int d = tid;
    uint32_t cnt = 0, c_incl = 0;
    if (d < R) {
#pragma unroll
        for (int ww = 0; ww < NW; ww++) {
            const uint32_t c = s_whist[ww][d];
            s_whist[ww][d] = (uint16_t)cnt;
            cnt += c;
        }
        if (a.late && !nolb) put_status(a.status, S32, (uint64_t)tile * R + d, tile == 0 ? kFlagP : kFlagA, cnt);
        c_incl = cnt;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const uint32_t cv = __shfl_up_sync(0xffffffffu, c_incl, o);
            if (lane >= o) c_incl += cv;
        }
        if (lane == 31) s_cw[w] = c_incl;
    }
    __syncthreads();
    if (d < R) {
        uint32_t coff = 0;
        for (int ww = 0; ww < w; ww++) coff += s_cw[ww];
        const uint32_t c_excl = coff + c_incl - cnt;
        s_lstart[d] = c_excl;
        if (d == R - 1) s_lstart[R] = c_excl + cnt;
#if SR_SORT_LSMERGE
        // fold the tile offset into every warp's base: one lookup per key in the scatter
#pragma unroll
        for (int ww = 0; ww < NW; ww++) s_whist[ww][d] = (uint16_t)(s_whist[ww][d] + c_excl);
#endif
    }
    __syncthreads();

    // scatter into shared memory in tile-sorted order (needs only local
    // offsets: predecessors keep publishing meanwhile)
#pragma unroll
    for (int j = 0; j < IT; j++) {
        const uint64_t i = wbase + (uint64_t)j * 32 + lane;
        if (FULL || i < a.n) {
            const uint32_t dd = (uint32_t)(key[j] >> a.shift) & (R - 1);
#if SR_SORT_LSMERGE
            const uint32_t lp = s_whist[w][dd] + ((rank2[j / 2] >> (16 * (j & 1))) & 0xffffu);
#else
            const uint32_t lp = s_lstart[dd] + s_whist[w][dd] + ((rank2[j / 2] >> (16 * (j & 1))) & 0xffffu);
#endif
            SR_DCHECK(lp < (uint32_t)TILE);
            s_keys[lp] = key[j];
            if (!PK) s_vals[lp] = val[PK ? 0 : j];
        }
    }

    // decoupled look-back (thread d < R owns digit d), kLB predecessors per
    // round trip; global offset = pass digit base + predecessors' counts
    if (d < R) {
        uint64_t excl = 0;
#ifdef SR_SORT_FAKE_LB   // timing experiment only (tools/sortbench): no look-back, approximate offsets, wrong output
        excl = (uint64_t)((double)a.hist[a.pass * kHistR + d] * tile / (double)((a.n + TILE - 1) / TILE));
        if (false) {
#else
        if (nolb) excl = a.tile_excl[(uint64_t)tile * R + d];
        if (tile != 0 && !nolb) {
#endif
            int64_t j = (int64_t)tile - 1;
            bool done = false;
            while (!done) {
                uint64_t sv[kLB];
#pragma unroll
                for (int q = 0; q < kLB; q++)
                    sv[q] = (j - q >= 0) ? get_status(a.status, S32, (uint64_t)(j - q) * R + d) : kFlagP;
#pragma unroll
                for (int q = 0; q < kLB; q++) {
                    if (done) break;
                    const uint64_t v = sv[q];
                    if (v & kFlagP) { excl += v & kValMask; done = true; }
                    else if (v & kFlagA) { excl += v & kValMask; j--; }
                    else { if (a.nap) __nanosleep(a.nap); break; }   // not published yet: poll again from tile j
                }
            }
            put_status(a.status, S32, (uint64_t)tile * R + d, kFlagP, excl + cnt);
        }
        s_delta[d] = (uint32_t)(a.gbase[a.pass * kHistR + d] + excl) - s_lstart[d];
    }
    __syncthreads();
    const uint32_t nvalid = s_lstart[R];
#pragma unroll 4
    for (uint32_t i = tid; i < nvalid; i += NT) {
        const uint64_t k = s_keys[i];
        const uint32_t dd = (uint32_t)(k >> a.shift) & (R - 1);
        uint32_t gp = s_delta[dd] + i;
        SR_DCHECK(gp < a.n);
#ifdef SR_SORT_FAKE_LB
        if (gp >= a.n) gp = (uint32_t)(a.n - 1);
#endif
        if (LAST) {
            const uint64_t kk = PK ? k >> a.ks : k;
            const uint32_t g = a.tab ? __ldg(a.tab + (kk >> a.tsh))
                                     : (uint32_t)(upper_bound(a.B, (uint64_t)a.K + 1, kk) - 1);
            __stcs(a.t_out + gp, (uint32_t)(kk - __ldg(a.B + g)));
            __stcs(a.row_out + gp, PK ? (uint32_t)(k & a.lomask) : s_vals[i]);
        } else {
            __stcs(a.keys_out + gp, k);
            if (!PK) __stcs(a.vals_out + gp, s_vals[i]);
        }
    }
}

// ---------------------------------------------------------------- host driver
// resident blocks per SM the first pass leaves L1 room for (its B[kid] gather
// table lives in L1); STEMROOT_FIRST_BLOCKS overrides
static int first_blocks() {
    static int v = -1;
    if (v < 0) {
        const char *e = getenv("STEMROOT_FIRST_BLOCKS");
        v = e ? atoi(e) : 3;
        if (v < 1 || v > 4) v = 3;
    }
    return v;
}

// full tiles in one launch (no bounds checks), the ragged last tile in a second
// launch: its look-back finds every predecessor already inclusive
template <int NT, int IT, bool FIRST, bool LAST, bool PK, bool S32>
static int launch_pass(const PassArgs &a, cudaStream_t st, uint32_t *launches) {
    constexpr uint64_t TILE = (uint64_t)NT * IT;
    const uint64_t full = a.n / TILE, rag = a.n % TILE;
    const size_t smem = (size_t)TILE * (sizeof(uint64_t) + (PK ? 0 : sizeof(uint32_t))) + sizeof(uint16_t) * (NT / 32) * kR +
                        (FIRST ? sizeof(uint32_t) * kR * (size_t)a.nxh : 0);
    // attributes once per instantiation (thread-safe static init: ranks of a
    // loopback group launch from several host threads), sized for the largest
    // dynamic shared memory any call can ask for (FIRST: kMaxPasses - 2 extra histograms)
    static const int attr_status = [] {
        const size_t smax = (size_t)TILE * (sizeof(uint64_t) + (PK ? 0 : sizeof(uint32_t))) +
                            sizeof(uint16_t) * (NT / 32) * kR + (FIRST ? sizeof(uint32_t) * kR * (kMaxPasses - 2) : 0);
        const size_t sbase = smax - (FIRST ? sizeof(uint32_t) * kR * (kMaxPasses - 2) : 0);
        // FIRST gathers B[kid]: keep L1 beside first_blocks() blocks' shared memory
        const int carve = FIRST ? (int)((first_blocks() * (sbase + 12 * 1024) * 100 + 228 * 1024 - 1) / (228 * 1024)) : 100;
        for (int f = 0; f < 2; f++) {
            auto fn = f ? onesweep_kernel<NT, IT, FIRST, LAST, true, PK, S32>
                        : onesweep_kernel<NT, IT, FIRST, LAST, false, PK, S32>;
            if (cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smax) != cudaSuccess ||
                cudaFuncSetAttribute(fn, cudaFuncAttributePreferredSharedMemoryCarveout, carve > 100 ? 100 : carve) !=
                    cudaSuccess)
                return 1;
        }
        return 0;
    }();
    if (attr_status) return STEM_E_CUDA;
    if (full) {
        onesweep_kernel<NT, IT, FIRST, LAST, true, PK, S32><<<(unsigned)full, NT, smem, st>>>(a);
        (*launches)++;
    }
    if (rag) {
        PassArgs ar = a;
        ar.tile_base = full;   // (tile_excl: the ragged tile's index)
        onesweep_kernel<NT, IT, FIRST, LAST, false, PK, S32><<<1, NT, smem, st>>>(ar);
        (*launches)++;
    }
    return STEM_OK;
}

template <int NT, int IT, bool PK, bool S32>
static int launch_pass_pk(const PassArgs &a, bool first, bool last, cudaStream_t st, uint32_t *launches) {
    if (first && last) return launch_pass<NT, IT, true, true, PK, S32>(a, st, launches);
    if (first) return launch_pass<NT, IT, true, false, PK, S32>(a, st, launches);
    if (last) return launch_pass<NT, IT, false, true, PK, S32>(a, st, launches);
    return launch_pass<NT, IT, false, false, PK, S32>(a, st, launches);
}

template <int NT, int IT>
static int launch_pass_cfg(const PassArgs &a, bool first, bool last, cudaStream_t st, uint32_t *launches) {
    // 32-bit look-back statuses only in the packed mode (the common one); the
    // payload mode keeps 64-bit ones
    if (!a.ks) return launch_pass_pk<NT, IT, false, false>(a, first, last, st, launches);
    return a.s32 ? launch_pass_pk<NT, IT, true, true>(a, first, last, st, launches)
                 : launch_pass_pk<NT, IT, true, false>(a, first, last, st, launches);
}

// tile shape (threads, keys per thread): 256 x 20 (4 blocks/SM) measured
// fastest on B200 for packed keys (C5 mid pass 5.07 ms vs 5.36 for 384 x 12,
// 5.09-5.29 for 256 x 16/24; the other shapes were dropped after the sweep)
constexpr int kSortNT = 256, kSortIT = 20;
static uint64_t tile_keys() { return (uint64_t)kSortNT * kSortIT; }

static int launch_sort_pass(const PassArgs &a, bool first, bool last, cudaStream_t st, uint32_t *launches) {
    return launch_pass_cfg<kSortNT, kSortIT>(a, first, last, st, launches);
}

// the pre-pass alone (kernel-id counts and max t, range check): also the
// multi-GPU histogram step.  Zeroes its outputs first (zero = false: they
// accumulate, for a trace handed over in chunks; pst = the launch stream).
int histogram_kernels(Ctx &c, const uint32_t *kid, const uint32_t *t, uint64_t n, uint32_t K, uint32_t *tailh,
                      bool zero, cudaStream_t pst, uint16_t *tileh, uint64_t tile0) {
    cudaStream_t st = pst ? pst : c.stream;
    if (zero) {
        CK(cudaMemsetAsync(c.hist, 0, sizeof(uint64_t) * (kMaxPasses + 1) * kHistR, st));
        if (tailh) CK(cudaMemsetAsync(tailh, 0, sizeof(uint32_t) * kR * (uint64_t)K, st));
        CK(cudaMemsetAsync(c.kid_count, 0, sizeof(uint32_t) * ((uint64_t)K + 1), st));
        CK(cudaMemsetAsync(c.kid_max, 0, sizeof(uint32_t) * ((uint64_t)K + 1), st));
    }
    if (n == 0) return STEM_OK;
    const int smem_kid = (K <= 24000) ? 1 : 0;
    static const int wtile = !(getenv("STEMROOT_PRE_WTILE") && getenv("STEMROOT_PRE_WTILE")[0] == '0');
    if (tileh && wtile) {   // tiles dealt to warps (default)
        const size_t tb = sizeof(uint32_t) * (3 * kR + 32 * (kR / 2) + (smem_kid ? 2 * (size_t)K : 0));
        static const cudaError_t pw_attr = cudaFuncSetAttribute(
            prepass_wtile_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
            (int)(sizeof(uint32_t) * (3 * kR + 32 * (kR / 2) + 2 * 24000)));
        CK(pw_attr);
        int per_sm = (int)((220 * 1024) / (tb + 1024));
        per_sm = per_sm < 1 ? 1 : per_sm > 2 ? 2 : per_sm;
        prepass_wtile_kernel<<<c.sms * per_sm, 1024, tb, st>>>(kid, t, n, K, smem_kid, c.kid_count, c.kid_max, c.hist,
                                                                &c.scalars->max_t, &c.scalars->err, tailh, tileh, tile0,
                                                                (uint32_t)tile_keys());
        c.launches++;
        CK(cudaGetLastError());
        return STEM_OK;
    }
    if (tileh) {   // whole sort tiles, with the first pass's per-tile digit histograms
        const size_t tb = sizeof(uint32_t) * ((3 + kPreTiles) * kR + (smem_kid ? 2 * (size_t)K : 0));
        static const cudaError_t pt_attr = cudaFuncSetAttribute(
            prepass_tile_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
            (int)(sizeof(uint32_t) * ((3 + kPreTiles) * kR + 2 * 24000)));
        CK(pt_attr);
        int per_sm = (int)((220 * 1024) / (tb + 1024));
        per_sm = per_sm < 1 ? 1 : per_sm > SR_PRET_MINB ? SR_PRET_MINB : per_sm;   // the registers allow SR_PRET_MINB
        prepass_tile_kernel<<<c.sms * per_sm, kPreTThreads, tb, st>>>(kid, t, n, K, smem_kid, c.kid_count, c.kid_max,
                                                                      c.hist, &c.scalars->max_t, &c.scalars->err, tailh,
                                                                      tileh, tile0, (uint32_t)tile_keys());
        c.launches++;
        CK(cudaGetLastError());
        return STEM_OK;
    }
    constexpr int kMaxNC = 8;
    auto bytes = [&](int nc) { return sizeof(uint32_t) * (nc * (3 * kR + 1) + (smem_kid ? 2 * (size_t)K : 0)); };
    // histogram copies (env STEMROOT_PRE_NC, <= 8, capped to keep two blocks per SM).
    // Default 1: on C5 the pre-pass takes 1.98 / 2.08 / 2.16 ms with 1 / 2 / 4 copies
    // (the extra shared memory and final reduction cost more than the rarer collisions)
    int nc = 1;
    if (const char *e = getenv("STEMROOT_PRE_NC")) nc = atoi(e);
    nc = nc < 1 ? 1 : nc > kMaxNC ? kMaxNC : nc;
    while (nc > 1 && ((nc & (nc - 1)) || 2 * (bytes(nc) + 1024) > 200 * 1024)) nc--;
    const size_t sm_bytes = bytes(nc);
    // once, for the largest request (thread-safe: loopback ranks are host threads)
    static const cudaError_t pre_attr = cudaFuncSetAttribute(
        prepass_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
        (int)(sizeof(uint32_t) * (kMaxNC * (3 * kR + 1) + 2 * 24000)));
    CK(pre_attr);
    int per_sm = (int)((200 * 1024) / (sm_bytes + 1024));
    per_sm = per_sm < 1 ? 1 : per_sm > 2 ? 2 : per_sm;
    prepass_kernel<<<c.sms * per_sm, kPreThreads, sm_bytes, st>>>(kid, t, n, K, smem_kid, c.kid_count, c.kid_max, c.hist,
                                                          &c.scalars->max_t, &c.scalars->err, tailh, nc);
    c.launches++;
    CK(cudaGetLastError());
    return STEM_OK;
}

// chunks of a host trace's copy (pre-pass overlapped with the copy); STEMROOT_H2D_CHUNKS
static int h2d_chunks(uint64_t n) {
    static int v = -1;
    if (v < 0) {
        const char *e = getenv("STEMROOT_H2D_CHUNKS");
        v = e ? atoi(e) : 8;
        v = v < 1 ? 1 : v > 8 ? 8 : v;
    }
    return n >= (1ull << 24) ? v : 1;
}

int sort_trace(Ctx &c, const uint32_t *kid, const uint32_t *t, const uint32_t *row_in, uint64_t n, uint32_t K,
               bool allow_pack, const uint32_t *h_kid, const uint32_t *h_t) {
    cudaStream_t st = c.stream;
    CK(cudaMemsetAsync(c.scalars, 0, sizeof(DevScalars), st));
    // coarse bases are possible when the [K][256] tail histogram is small
    const bool coarse_ok = K <= kMaxTailK && !(getenv("STEMROOT_SORT_COARSE") && getenv("STEMROOT_SORT_COARSE")[0] == '0');
    if (coarse_ok) CKS(c.ensure(c.tailh, c.cap_tailh, sizeof(uint32_t) * kR * (uint64_t)K));
    uint32_t *tailh = coarse_ok ? c.tailh : nullptr;
    // the first pass without look-back: the pre-pass counts its digit per tile
    // and three small kernels turn the counts into each tile's offsets
    // (STEMROOT_SORT_NOLB=0: the look-back first pass)
    const uint64_t ntiles = (n + tile_keys() - 1) / tile_keys();
    const bool nolb = !(getenv("STEMROOT_SORT_NOLB") && getenv("STEMROOT_SORT_NOLB")[0] == '0') && n > 0;
    const uint64_t ngrp = (ntiles + kExGrp - 1) / kExGrp;
    uint16_t *tileh = nullptr;
    uint32_t *tgrp = nullptr, *texcl = nullptr;
    if (nolb) {
        const size_t b_h = (sizeof(uint16_t) * ntiles * kR + 255) & ~(size_t)255;
        const size_t b_g = (sizeof(uint32_t) * ngrp * kR + 255) & ~(size_t)255;
        CKS(c.ensure(c.tile_hist, c.cap_tile_hist, b_h + b_g + sizeof(uint32_t) * ntiles * kR));
        tileh = (uint16_t *)c.tile_hist;
        tgrp = (uint32_t *)((char *)c.tile_hist + b_h);
        texcl = (uint32_t *)((char *)c.tile_hist + b_h + b_g);
    }
    const int nch = h_kid ? h2d_chunks(n) : 0;
    if (nch > 1) {
        // host trace: the copies run back to back on the plan's stream; the
        // pre-pass of chunk i runs on dstream as soon as chunk i has landed
        if (!c.dstream) {
            CK(cudaStreamCreateWithFlags(&c.dstream, cudaStreamNonBlocking));
            CK(cudaEventCreateWithFlags(&c.ev_pack, cudaEventDisableTiming));
            CK(cudaEventCreateWithFlags(&c.ev_d2h, cudaEventDisableTiming));
        }
        for (int i = 0; i < nch; i++)
            if (!c.ev_h2d[i]) CK(cudaEventCreateWithFlags(&c.ev_h2d[i], cudaEventDisableTiming));
        if (!c.ev_pre) CK(cudaEventCreateWithFlags(&c.ev_pre, cudaEventDisableTiming));
        CKS(histogram_kernels(c, nullptr, nullptr, 0, K, tailh, true, st));   // zero the outputs
        const uint64_t step = ((n + nch - 1) / nch + tile_keys() - 1) / tile_keys() * tile_keys();   // whole tiles
        int used = 0;
        for (uint64_t r0 = 0; r0 < n; r0 += step, used++) {
            const uint64_t cnt = min(step, n - r0);
            CK(cudaMemcpyAsync((void *)(kid + r0), h_kid + r0, sizeof(uint32_t) * cnt, cudaMemcpyHostToDevice, st));
            CK(cudaMemcpyAsync((void *)(t + r0), h_t + r0, sizeof(uint32_t) * cnt, cudaMemcpyHostToDevice, st));
            CK(cudaEventRecord(c.ev_h2d[used], st));
            CK(cudaStreamWaitEvent(c.dstream, c.ev_h2d[used], 0));
            CKS(histogram_kernels(c, kid + r0, t + r0, cnt, K, tailh, false, c.dstream, tileh, r0 / tile_keys()));
        }
        CK(cudaEventRecord(c.ev_pre, c.dstream));
        CK(cudaStreamWaitEvent(st, c.ev_pre, 0));
    } else if (h_kid) {
        CK(cudaMemcpyAsync((void *)kid, h_kid, sizeof(uint32_t) * n, cudaMemcpyHostToDevice, st));
        CK(cudaMemcpyAsync((void *)t, h_t, sizeof(uint32_t) * n, cudaMemcpyHostToDevice, st));
    }
    const int tk_pre = c.stage_begin("prepass");
    if (nch <= 1) CKS(histogram_kernels(c, kid, t, n, K, tailh, true, st, tileh, 0));
    if (nolb) {
        tile_grp_kernel<<<(unsigned)ngrp, kR, 0, st>>>(tileh, ntiles, tgrp);
        grp_scan_kernel<<<kR, 1024, 0, st>>>(tgrp, ngrp);
        tile_excl_kernel<<<(unsigned)ngrp, kR, 0, st>>>(tileh, ntiles, tgrp, texcl);
        c.launches += 3;
    }
    // key bases B = exclusive scan of W[k] = roundup(max_t[k] + 1, 2^16) (0 if
    // absent); Bc the same with 2^24
    const uint32_t *cnt = c.kid_count, *kmax = c.kid_max;
    for (int v = 0; v < (coarse_ok ? 2 : 1); v++) {
        uint64_t *Bv = v ? c.key_base_c : c.key_base;
        const int sh = v ? kCoarseShift : kBaseShift;
        exclusive_scan<uint64_t>(
            [cnt, kmax, K, sh] __device__(uint64_t i) -> uint64_t {
                if (i >= K || cnt[i] == 0) return 0;
                return (((uint64_t)kmax[i] >> sh) + 1) << sh;
            },
            [Bv] __device__(uint64_t i, uint64_t pre, uint64_t) { Bv[i] = pre; }, (uint64_t)K + 1,
            (uint64_t *)c.scan_scratch, v ? &c.scalars->scan_total64b : &c.scalars->scan_total64, st, &c.launches);
    }
    DevScalars hs;
    CK(cudaMemcpyAsync(&hs, c.scalars, sizeof(DevScalars), cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
    if (hs.err) return STEM_E_RANGE;
    auto nbits = [](uint64_t range) {   // keys lie in [0, range)
        int b = 0;
        while (b < 64 && (b == 0 || (range - 1) >> b)) b++;
        return b;
    };
    auto npass = [](int b) { return b <= 16 ? 2 : (b + kRB - 1) / kRB; };
    int bits = nbits(hs.scan_total64);
    bool coarse = false;
    if (coarse_ok && hs.scan_total64b && npass(nbits(hs.scan_total64b)) <= npass(bits)) {
        coarse = true;
        bits = nbits(hs.scan_total64b);
    }
    const uint64_t range = coarse ? hs.scan_total64b : hs.scan_total64;
    const int npasses = npass(bits);
    if (npasses > kMaxPasses) return STEM_E_RANGE;
    uint64_t *B = coarse ? c.key_base_c : c.key_base;
    if (coarse) {
        coarse_hist_kernel<<<(unsigned)((K + 7) / 8), kR, 0, st>>>(cnt, c.tailh, B, K, npasses, n, c.hist);
        c.launches++;
    }
    c.stage_end(tk_pre, 8 * n);
    c.stats.coarse_bases = coarse ? 1 : 0;
    c.stats.key_bits = bits;
    c.stats.sort_passes = npasses;
    // packed mode: s = 64 - bits low row bits in the key, at most kMaxCand
    // candidate rows per sample (STEMROOT_SORT_PACK=0 forces the payload mode,
    // STEMROOT_PACK_BITS=s a smaller s, for tests of the candidate path)
    int ks = 64 - bits;
    if (const char *e = getenv("STEMROOT_PACK_BITS")) {
        const int f = atoi(e);
        if (f > 0 && f < ks) ks = f;
    }
    uint64_t hcount = 1;
    if (ks < 32) hcount = (n + (1ull << ks) - 1) >> ks;
    if (const char *e = getenv("STEMROOT_SORT_PACK"))
        if (e[0] == '0') allow_pack = false;
    if (!allow_pack || ks <= 0 || hcount > (uint64_t)kMaxCand) ks = 0;
    c.pack_s = ks;
    c.pack_h = ks ? (uint32_t)hcount : 0;
    c.sort_kid = kid;
    c.sort_t = t;
    c.sort_row_in = row_in;
    c.stats.pack_bits = (uint32_t)ks;

    // kid table for the last pass
    const int tsh = coarse ? kCoarseShift : kBaseShift;
    const uint64_t entries = range >> tsh;
    const uint32_t *tab = nullptr;
    if (entries <= kMaxTable) {
        CKS(c.ensure(c.kid_tab, c.cap_kid_tab, sizeof(uint32_t) * (entries + 1)));
        kid_table_kernel<<<(unsigned)((entries + 255) / 256), 256, 0, st>>>(B, K, entries, tsh, c.kid_tab);
        c.launches++;
        tab = c.kid_tab;
    }

    CKS(c.ensure(c.sort_status, c.cap_status, ntiles * kR * sizeof(uint64_t)));
    PassArgs a{};
    a.n = n;
    a.K = K;
    a.B = B;
    a.Bs = nullptr;
    a.Bs16 = nullptr;
    if ((range >> tsh) < (1ull << 32)) {   // bases >> tsh fit 32 (or 16) bits
        const bool b16 = (range >> tsh) < (1ull << 16) && !(getenv("STEMROOT_SORT_BS16") && getenv("STEMROOT_SORT_BS16")[0] == '0');
        CKS(c.ensure(c.key_base_s, c.cap_kbase_s, sizeof(uint32_t) * ((uint64_t)K + 2)));
        base_shift_kernel<<<(unsigned)((K + 256) / 256), 256, 0, st>>>(B, (uint64_t)K + 1, tsh, b16 ? nullptr : c.key_base_s,
                                                                       b16 ? (uint16_t *)c.key_base_s : nullptr);
        c.launches++;
        if (b16) a.Bs16 = (const uint16_t *)c.key_base_s;
        else a.Bs = c.key_base_s;
    }
    a.tab = tab;
    a.nxh = coarse ? 0 : npasses - 2;
    a.tsh = tsh;
    a.ks = ks;
    a.lomask = ks ? (ks >= 32 ? 0xffffffffull : (1ull << ks) - 1) : 0;
    {
        static int pf = -1;
        if (pf < 0) {
            const char *e = getenv("STEMROOT_SORT_PF");
            pf = e ? atoi(e) : 3 * c.sms;   // about one wave of resident tiles (measured best)
        }
        a.pf = (uint32_t)pf;
    }
    a.nap = 20;
    if (const char *e = getenv("STEMROOT_SORT_NAP")) a.nap = (uint32_t)atoi(e);
    // publish the tile's counts after ranking (from the warp histograms): no
    // separate counting of the keys (C5 mid pass 4.67 ms vs 4.94 counting first)
    a.late = 1;
    a.noalloc = 1;
    if (const char *e = getenv("STEMROOT_SORT_NOALLOC")) a.noalloc = atoi(e) ? 1 : 0;
    if (const char *e = getenv("STEMROOT_SORT_LATE")) a.late = atoi(e) ? 1 : 0;
    int late_first = a.late;   // STEMROOT_SORT_LATE_FIRST: the first pass's publication alone
    if (const char *e = getenv("STEMROOT_SORT_LATE_FIRST")) late_first = atoi(e) ? 1 : 0;
    const int late_rest = a.late;
    int rank_force = -1;   // STEMROOT_SORT_RANK=match|ballot forces one ranking mode
    double rank_thr = 24.0;   // STEMROOT_SORT_RANK_THR: ballots from this many expected distinct digits
    if (const char *e = getenv("STEMROOT_SORT_RANK_THR")) rank_thr = atof(e);
    if (const char *e = getenv("STEMROOT_SORT_RANK")) rank_force = e[0] == 'b' ? 1 : e[0] == 'm' ? 0 : -1;
    uint32_t *mode = c.sort_mode;
    uint64_t *gbase = c.sort_gbase;
    rank_mode_kernel<<<1, kR, 0, st>>>(c.hist, 0, 2, n, rank_force, rank_thr, mode, gbase);   // key bytes 0, 1: pre-pass
    c.launches++;
    a.ballot = mode;
    a.gbase = gbase;
    a.hist = c.hist;
    a.status = (uint64_t *)c.sort_status;
    a.s32 = ks && n < (1ull << 30) && !(getenv("STEMROOT_SORT_S32") && getenv("STEMROOT_SORT_S32")[0] == '0');
    const size_t status_bytes = ntiles * kR * (a.s32 ? sizeof(uint32_t) : sizeof(uint64_t));
    a.tile_counter = &c.scalars->tile_counter;
    uint64_t *kin = c.keys[0], *kout = c.keys[1];
    uint32_t *vin = c.vals[0], *vout = c.vals[1];
    for (int p = 0; p < npasses; p++) {
        a.tile_excl = p == 0 && nolb ? texcl : nullptr;
        a.tile_base = 0;
        if (!a.tile_excl) {
            CK(cudaMemsetAsync(a.status, 0, status_bytes, st));
            CK(cudaMemsetAsync(a.tile_counter, 0, sizeof(uint32_t), st));
        }
        a.shift = ks + kRB * p;
        a.pass = p;
        const bool first = p == 0, last = p == npasses - 1;
        a.late = first ? late_first : late_rest;
        a.kid_in = kid;
        a.t_in = t;
        a.row_in = row_in;
        a.keys_in = kin;
        a.vals_in = vin;
        a.keys_out = kout;
        a.vals_out = vout;
        a.t_out = c.t_sorted;
        a.row_out = c.row_sorted;
        const char *sname = first ? "sort_pass_first" : last ? "sort_pass_last" : "sort_pass_mid";
        const uint64_t sbytes = n * ((first ? 8 : ks ? 8 : 12) + (last ? 8 : ks ? 8 : 12));
        const int tk = c.stage_begin(sname);
        CKS(launch_sort_pass(a, first, last, st, &c.launches));
        c.stage_end(tk, sbytes);
        CK(cudaGetLastError());
        if (first && npasses > 2) {   // higher bytes: histogrammed by pass 0
            rank_mode_kernel<<<1, kR, 0, st>>>(c.hist, 2, npasses, n, rank_force, rank_thr, mode, gbase);
            c.launches++;
        }
        uint64_t *tkk = kin; kin = kout; kout = tkk;
        uint32_t *tv = vin; vin = vout; vout = tv;
    }
    // group offsets: goff = exclusive scan of kernel counts
    uint32_t *goff = c.goff;
    const int tk_g = c.stage_begin("group_offsets");
    exclusive_scan<uint64_t>(
        [cnt, K] __device__(uint64_t i) -> uint64_t { return i < K ? (uint64_t)cnt[i] : 0; },
        [goff] __device__(uint64_t i, uint64_t pre, uint64_t) { goff[i] = (uint32_t)pre; },
        (uint64_t)K + 1, (uint64_t *)c.scan_scratch, &c.scalars->scan_total64, st, &c.launches);
    c.stage_end(tk_g, 8 * ((uint64_t)K + 1));
    CK(cudaGetLastError());
    return STEM_OK;
}

}  // namespace sr
