// sort.cu -- step a1 (group by kernel): stable LSD radix sort of the
// packed key (kernel_id << tbits | t) carrying the trace row, one-sweep style
// (Adinets & Merrill): every pass reads and writes the data once, tiles get
// their global digit offsets by decoupled look-back.  The pre-pass validates
// kernel ids, finds max t, histograms kernel ids (group sizes) and digit 0;
// pass 0 histograms all later digits, so no extra histogram pass is needed.
#include <cstdlib>

#include "internal.h"

namespace sr {

constexpr int kRadix = 256;
constexpr uint64_t kFlagA = 1ull << 62, kFlagP = 2ull << 62, kValMask = (1ull << 62) - 1;

// ---------------------------------------------------------------- pre-pass
__global__ void __launch_bounds__(256) prepass_kernel(const uint32_t *__restrict__ kid, const uint32_t *__restrict__ t,
                                                      uint64_t n, uint32_t K, int smem_kid_hist,
                                                      uint32_t *__restrict__ kid_count, uint64_t *__restrict__ hist_t,
                                                      uint32_t *__restrict__ max_t, uint32_t *__restrict__ err) {
    extern __shared__ uint32_t sh[];   // [4][256] histograms of the 4 bytes of t, then [K] kernel hist
    uint32_t *h0 = sh, *hk = sh + 4 * kRadix;
    for (int i = threadIdx.x; i < 4 * kRadix; i += blockDim.x) h0[i] = 0;
    if (smem_kid_hist)
        for (uint32_t i = threadIdx.x; i < K; i += blockDim.x) hk[i] = 0;
    __syncthreads();
    uint32_t mx = 0, bad = 0;
    const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    const uint64_t n4 = n / 4;
    const uint4 *kid4 = reinterpret_cast<const uint4 *>(kid), *t4 = reinterpret_cast<const uint4 *>(t);
    auto one = [&](uint32_t k, uint32_t x) {
        mx = max(mx, x);
        atomicAdd(&h0[x & 0xFF], 1u);
        atomicAdd(&h0[kRadix + ((x >> 8) & 0xFF)], 1u);
        atomicAdd(&h0[2 * kRadix + ((x >> 16) & 0xFF)], 1u);
        atomicAdd(&h0[3 * kRadix + (x >> 24)], 1u);
        if (k >= K) { bad = 1; return; }
        if (smem_kid_hist) atomicAdd(&hk[k], 1u); else atomicAdd(&kid_count[k], 1u);
    };
    const bool aligned = ((reinterpret_cast<uintptr_t>(kid) | reinterpret_cast<uintptr_t>(t)) & 15) == 0;
    if (aligned) {
        for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n4; i += stride) {
            const uint4 a = __ldg(kid4 + i), b = __ldg(t4 + i);
            one(a.x, b.x); one(a.y, b.y); one(a.z, b.z); one(a.w, b.w);
        }
        for (uint64_t i = n4 * 4 + (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += stride)
            one(__ldg(kid + i), __ldg(t + i));
    } else {
        for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += stride)
            one(__ldg(kid + i), __ldg(t + i));
    }
    // reductions
    for (int o = 16; o; o >>= 1) {
        mx = max(mx, __shfl_xor_sync(0xffffffffu, mx, o));
        bad |= __shfl_xor_sync(0xffffffffu, bad, o);
    }
    if ((threadIdx.x & 31) == 0) {
        if (mx) atomicMax(max_t, mx);
        if (bad) atomicOr(err, 1u);
    }
    __syncthreads();
    for (int i = threadIdx.x; i < 4 * kRadix; i += blockDim.x)
        if (h0[i]) atomicAdd((unsigned long long *)&hist_t[i], (unsigned long long)h0[i]);
    if (smem_kid_hist)
        for (uint32_t i = threadIdx.x; i < K; i += blockDim.x)
            if (hk[i]) atomicAdd(&kid_count[i], hk[i]);
}

// histograms of the kernel-id bytes of the aligned key, from the kernel-id counts
__global__ void kid_digit_hist_kernel(const uint32_t *__restrict__ kid_count, uint32_t K, int nbytes,
                                      uint64_t *__restrict__ hist) {
    const uint64_t g = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (g >= K || kid_count[g] == 0) return;
    for (int b = 0; b < nbytes; b++)
        atomicAdd((unsigned long long *)&hist[b * kRadix + ((g >> (8 * b)) & 0xFF)], (unsigned long long)kid_count[g]);
}

// ---------------------------------------------------------------- one-sweep pass
struct PassArgs {
    const uint32_t *kid_in, *t_in;      // FIRST: trace columns
    const uint32_t *row_in;             // FIRST: row payload (NULL = the row index)
    const uint64_t *keys_in;            // !FIRST
    const uint32_t *vals_in;            // !FIRST
    uint64_t *keys_out;                 // !LAST
    uint32_t *vals_out;                 // !LAST
    uint32_t *t_out, *row_out;          // LAST
    uint64_t n;
    int shift, tbits, npasses;
    int first_hist;                     // FIRST: accumulate the later digits' histograms here
    const uint64_t *hist;               // [npasses][256] global digit counts
    uint64_t *hist_all;                 // FIRST: accumulates digits 1..npasses-1
    uint64_t *status;                   // [ntiles][256]
    uint32_t *tile_counter;
};

// One LSD pass over 8-bit digit (key >> shift) & 0xFF.  NT threads, IT keys per
// thread, tile = NT*IT keys.  Keys are loaded warp-striped (coalesced), ranked
// in element order by warp-level multi-split (match.any), the tile's digit
// counts are published and the global offsets found by decoupled look-back
// (thread d < 256 owns digit d), then keys are staged in shared memory in
// tile-sorted order and written out in digit runs (coalesced).
template <int NT, int IT, bool FIRST, bool LAST>
__global__ void __launch_bounds__(NT, (NT >= 512 ? 2 : NT >= 384 ? 3 : NT >= 256 ? 4 : 8)) onesweep_kernel(PassArgs a) {
    constexpr int NW = NT / 32, TILE = NT * IT;
    extern __shared__ __align__(16) unsigned char s_dyn[];
    uint64_t *s_keys = reinterpret_cast<uint64_t *>(s_dyn);                          // [TILE]
    uint32_t *s_vals = reinterpret_cast<uint32_t *>(s_keys + TILE);                  // [TILE]
    uint16_t (*s_whist)[kRadix] = reinterpret_cast<uint16_t (*)[kRadix]>(s_vals + TILE);   // [NW][radix]
    uint32_t (*s_hlater)[kRadix] = reinterpret_cast<uint32_t (*)[kRadix]>(s_whist + NW);   // FIRST: [7][radix]
    __shared__ uint64_t s_delta[kRadix];
    __shared__ uint32_t s_lstart[kRadix + 1];
    __shared__ uint64_t s_gw[8];
    __shared__ uint32_t s_cw[8];
    __shared__ uint32_t s_tile;
    __shared__ uint32_t s_cnt[kRadix];

    const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
    if (tid == 0) s_tile = atomicAdd(a.tile_counter, 1u);
    for (int i = tid; i < NW * kRadix / 2; i += NT) reinterpret_cast<uint32_t *>(&s_whist[0][0])[i] = 0;
    for (int i = tid; i < kRadix; i += NT) s_cnt[i] = 0;
    if (FIRST && a.first_hist)
        for (int i = tid; i < 7 * kRadix; i += NT) (&s_hlater[0][0])[i] = 0;
    __syncthreads();
    const uint32_t tile = s_tile;
    const uint64_t wbase = (uint64_t)tile * TILE + (uint64_t)w * (32 * IT);
    const uint64_t tmask = (a.tbits >= 64) ? ~0ull : ((1ull << a.tbits) - 1);

    // load (warp-striped: item j of lane l is element wbase + 32 j + l)
    uint64_t key[IT];
    uint32_t val[IT];
#pragma unroll
    for (int j = 0; j < IT; j++) {
        const uint64_t i = wbase + (uint64_t)j * 32 + lane;
        if (i < a.n) {
            if (FIRST) {
                key[j] = ((uint64_t)__ldg(a.kid_in + i) << a.tbits) | (uint64_t)__ldg(a.t_in + i);
                val[j] = a.row_in ? __ldg(a.row_in + i) : (uint32_t)i;
            } else {
                key[j] = __ldcs(a.keys_in + i);
                val[j] = __ldcs(a.vals_in + i);
            }
        } else {
            key[j] = ~0ull;
            val[j] = 0;
        }
    }
    if (FIRST && a.first_hist) {   // histograms of the later digits (each key seen exactly once here)
#pragma unroll
        for (int j = 0; j < IT; j++) {
            const uint64_t i = wbase + (uint64_t)j * 32 + lane;
            if (i < a.n)
                for (int p = 1; p < a.npasses; p++) atomicAdd(&s_hlater[p - 1][(key[j] >> (8 * p)) & 0xFF], 1u);
        }
    }

    // tile digit counts first, published at once (flag A) so that successors'
    // look-backs do not wait for this tile's ranking
#pragma unroll
    for (int j = 0; j < IT; j++)
        if (wbase + (uint64_t)j * 32 + lane < a.n) atomicAdd(&s_cnt[(uint32_t)(key[j] >> a.shift) & 0xFF], 1u);
    __syncthreads();
    if (tid < kRadix) __stcg(a.status + (uint64_t)tile * kRadix + tid, (tile == 0 ? kFlagP : kFlagA) | s_cnt[tid]);

    // warp-level multi-split ranking, in element order
    uint32_t rank[IT];
#pragma unroll
    for (int j = 0; j < IT; j++) {
        const uint64_t i = wbase + (uint64_t)j * 32 + lane;
        const bool valid = i < a.n;
        const uint32_t vmask = __ballot_sync(0xffffffffu, valid);
        if (valid) {
            const uint32_t d = (uint32_t)(key[j] >> a.shift) & 0xFF;
            const uint32_t peers = __match_any_sync(vmask, d);
            const uint32_t base = s_whist[w][d];
            const uint32_t below = __popc(peers & ((1u << lane) - 1));
            rank[j] = base + below;
            __syncwarp(vmask);
            if (below == 0) s_whist[w][d] = (uint16_t)(base + __popc(peers));
        }
        __syncwarp();
    }
    __syncthreads();

    // digit phase (threads d < 256): warp offsets, tile count, look-back
    const int d = tid;
    uint32_t cnt = 0;
    uint64_t excl = 0, gcount = 0, g_incl = 0;
    uint32_t c_incl = 0;
    if (d < kRadix) {
#pragma unroll
        for (int ww = 0; ww < NW; ww++) {
            const uint32_t c = s_whist[ww][d];
            s_whist[ww][d] = (uint16_t)cnt;
            cnt += c;
        }
        uint64_t *st = a.status + (uint64_t)tile * kRadix + d;
        if (tile != 0) {
            int64_t j = (int64_t)tile - 1;
            while (true) {
                const uint64_t sv = *(volatile uint64_t *)(a.status + (uint64_t)j * kRadix + d);
                if (sv & kFlagP) { excl += sv & kValMask; break; }
                if (sv & kFlagA) { excl += sv & kValMask; j--; }
            }
            __stcg(st, kFlagP | (excl + cnt));
        }
        gcount = a.hist[(a.shift / 8) * kRadix + d];
        g_incl = gcount;
        c_incl = cnt;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const uint64_t gv = __shfl_up_sync(0xffffffffu, g_incl, o);
            const uint32_t cv = __shfl_up_sync(0xffffffffu, c_incl, o);
            if (lane >= o) { g_incl += gv; c_incl += cv; }
        }
        if (lane == 31) { s_gw[w] = g_incl; s_cw[w] = c_incl; }
    }
    __syncthreads();
    if (d < kRadix) {
        uint64_t goff = 0;
        uint32_t coff = 0;
        for (int ww = 0; ww < w; ww++) { goff += s_gw[ww]; coff += s_cw[ww]; }
        const uint64_t g_excl = goff + g_incl - gcount;
        const uint32_t c_excl = coff + c_incl - cnt;
        s_lstart[d] = c_excl;
        s_delta[d] = g_excl + excl - c_excl;   // global position - local position
        if (d == kRadix - 1) s_lstart[kRadix] = c_excl + cnt;
        if (FIRST && a.first_hist) {
            for (int p = 1; p < a.npasses; p++) {
                const uint32_t h = s_hlater[p - 1][d];
                if (h) atomicAdd((unsigned long long *)&a.hist_all[p * kRadix + d], (unsigned long long)h);
            }
        }
    }
    __syncthreads();

    // scatter into shared memory in tile-sorted order
#pragma unroll
    for (int j = 0; j < IT; j++) {
        const uint64_t i = wbase + (uint64_t)j * 32 + lane;
        if (i < a.n) {
            const uint32_t dd = (uint32_t)(key[j] >> a.shift) & 0xFF;
            const uint32_t lp = s_lstart[dd] + s_whist[w][dd] + rank[j];
            s_keys[lp] = key[j];
            s_vals[lp] = val[j];
        }
    }
    __syncthreads();
    const uint32_t nvalid = s_lstart[kRadix];
#pragma unroll 4
    for (uint32_t i = tid; i < nvalid; i += NT) {
        const uint64_t k = s_keys[i];
        const uint32_t dd = (uint32_t)(k >> a.shift) & 0xFF;
        const uint64_t gp = s_delta[dd] + i;
        if (LAST) {
            __stcs(a.t_out + gp, (uint32_t)(k & tmask));
            __stcs(a.row_out + gp, s_vals[i]);
        } else {
            __stcs(a.keys_out + gp, k);
            __stcs(a.vals_out + gp, s_vals[i]);
        }
    }
}

// ---------------------------------------------------------------- persistent TMA pass
// Same algorithm as onesweep_kernel, but persistent blocks with two smem tile
// buffers: while tile i is ranked, looked back and scattered, the Tensor Memory
// Accelerator (cp.async.bulk) streams tile i+1 into the other buffer.  The
// buffer of tile i doubles as the scatter staging area once its keys sit in
// registers.
__device__ __forceinline__ uint32_t smem_u32(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }

__device__ __forceinline__ void mbar_init(uint64_t *bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count));
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t *bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t *bar, uint32_t phase) {
    asm volatile(
        "{\n .reg .pred p;\n WAIT_%=:\n"
        " mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
        " @!p bra WAIT_%=;\n}" ::"r"(smem_u32(bar)),
        "r"(phase)
        : "memory");
}
__device__ __forceinline__ void tma_load(void *dst, const void *src, uint32_t bytes, uint64_t *bar) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                     smem_u32(dst)),
                 "l"(src), "r"(bytes), "r"(smem_u32(bar))
                 : "memory");
}
__device__ __forceinline__ void fence_async_smem() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }

constexpr int kTmaThreads = 512, kTmaItems = 8, kTmaTile = kTmaThreads * kTmaItems;   // 4096 keys

// The TMA part of a tile covers its first (cnt & ~3) elements (whole 16-byte
// units, never past the end of an array); the <= 3 tail elements are read
// directly from global memory.
__device__ __forceinline__ uint64_t tma_elems(const PassArgs &a, uint32_t tile) {
    const uint64_t start = (uint64_t)tile * kTmaTile;
    return min((uint64_t)kTmaTile, a.n - start) & ~3ull;
}

template <bool FIRST>
__device__ __forceinline__ void tma_issue(const PassArgs &a, uint32_t tile, unsigned char *buf, uint64_t *bar) {
    const uint64_t start = (uint64_t)tile * kTmaTile;
    const uint32_t e = (uint32_t)tma_elems(a, tile);
    if (FIRST) {
        mbar_expect_tx(bar, 8 * e);
        if (e) {
            tma_load(buf, a.kid_in + start, 4 * e, bar);
            tma_load(buf + kTmaTile * 8, a.t_in + start, 4 * e, bar);
        }
    } else {
        mbar_expect_tx(bar, 12 * e);
        if (e) {
            tma_load(buf, a.keys_in + start, 8 * e, bar);
            tma_load(buf + kTmaTile * 8, a.vals_in + start, 4 * e, bar);
        }
    }
}

template <bool FIRST, bool LAST>
__global__ void __launch_bounds__(kTmaThreads, 2) onesweep_tma_kernel(PassArgs a, uint32_t ntiles) {
    constexpr int NT = kTmaThreads, IT = kTmaItems, TILE = kTmaTile, NW = NT / 32;
    constexpr int BUF = TILE * 12;                      // keys (8 B) then vals (4 B); FIRST: kid, t
    extern __shared__ __align__(128) unsigned char s_dyn[];
    unsigned char *bufs = s_dyn;                        // [2][BUF]
    uint16_t (*s_whist)[kRadix] = reinterpret_cast<uint16_t (*)[kRadix]>(s_dyn + 2 * BUF);
    __shared__ __align__(8) uint64_t s_bar[2];
    __shared__ uint64_t s_delta[kRadix];
    __shared__ uint32_t s_lstart[kRadix + 1];
    __shared__ uint64_t s_gw[8];
    __shared__ uint32_t s_cw[8];
    __shared__ uint32_t s_next;

    const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
    const uint64_t tmask = (a.tbits >= 64) ? ~0ull : ((1ull << a.tbits) - 1);
    if (tid == 0) {
        mbar_init(&s_bar[0], 1);
        mbar_init(&s_bar[1], 1);
        fence_async_smem();
        s_next = atomicAdd(a.tile_counter, 1u);
    }
    __syncthreads();
    uint32_t tile = s_next;
    if (tile >= ntiles) return;
    if (tid == 0) tma_issue<FIRST>(a, tile, bufs, &s_bar[0]);
    uint32_t phase[2] = {0, 0};
    int cur = 0;
    while (true) {
        unsigned char *buf = bufs + cur * BUF;
        for (int i = tid; i < NW * kRadix / 2; i += NT) reinterpret_cast<uint32_t *>(&s_whist[0][0])[i] = 0;
        mbar_wait(&s_bar[cur], phase[cur]);
        phase[cur] ^= 1;
        // keys of this tile into registers (warp-striped)
        const uint64_t tbase = (uint64_t)tile * TILE;
        const uint64_t te = tma_elems(a, tile);
        const int wb = w * 32 * IT;
        uint64_t key[IT];
        uint32_t val[IT];
#pragma unroll
        for (int j = 0; j < IT; j++) {
            const int li = wb + j * 32 + lane;
            const uint64_t i = tbase + li;
            if (i < a.n) {
                const bool sm = (uint64_t)li < te;
                if (FIRST) {
                    const uint32_t kk = sm ? reinterpret_cast<const uint32_t *>(buf)[li] : __ldg(a.kid_in + i);
                    const uint32_t tv = sm ? reinterpret_cast<const uint32_t *>(buf + TILE * 8)[li] : __ldg(a.t_in + i);
                    key[j] = ((uint64_t)kk << a.tbits) | tv;
                    val[j] = a.row_in ? __ldg(a.row_in + i) : (uint32_t)i;
                } else {
                    key[j] = sm ? reinterpret_cast<const uint64_t *>(buf)[li] : a.keys_in[i];
                    val[j] = sm ? reinterpret_cast<const uint32_t *>(buf + TILE * 8)[li] : a.vals_in[i];
                }
            } else {
                key[j] = ~0ull;
                val[j] = 0;
            }
        }
        __syncthreads();   // buffer `cur` is free (becomes the staging area); whist zeroed
        // prefetch the next tile into the other buffer
        if (tid == 0) {
            s_next = atomicAdd(a.tile_counter, 1u);
            if (s_next < ntiles) {
                fence_async_smem();
                tma_issue<FIRST>(a, s_next, bufs + (cur ^ 1) * BUF, &s_bar[cur ^ 1]);
            }
        }
        // warp-level multi-split ranking
        uint32_t rank[IT];
#pragma unroll
        for (int j = 0; j < IT; j++) {
            const uint64_t i = tbase + wb + j * 32 + lane;
            const bool valid = i < a.n;
            const uint32_t vmask = __ballot_sync(0xffffffffu, valid);
            if (valid) {
                const uint32_t d = (uint32_t)(key[j] >> a.shift) & 0xFF;
                const uint32_t peers = __match_any_sync(vmask, d);
                const uint32_t base = s_whist[w][d];
                const uint32_t below = __popc(peers & ((1u << lane) - 1));
                rank[j] = base + below;
                __syncwarp(vmask);
                if (below == 0) s_whist[w][d] = (uint16_t)(base + __popc(peers));
            }
            __syncwarp();
        }
        __syncthreads();
        const int d = tid;
        uint32_t cnt = 0, c_incl = 0;
        uint64_t excl = 0, gcount = 0, g_incl = 0;
        if (d < kRadix) {
#pragma unroll
            for (int ww = 0; ww < NW; ww++) {
                const uint32_t c = s_whist[ww][d];
                s_whist[ww][d] = (uint16_t)cnt;
                cnt += c;
            }
            uint64_t *st = a.status + (uint64_t)tile * kRadix + d;
            if (tile == 0) {
                __stcg(st, kFlagP | cnt);
            } else {
                __stcg(st, kFlagA | cnt);
                int64_t j = (int64_t)tile - 1;
                while (true) {
                    const uint64_t sv = *(volatile uint64_t *)(a.status + (uint64_t)j * kRadix + d);
                    if (sv & kFlagP) { excl += sv & kValMask; break; }
                    if (sv & kFlagA) { excl += sv & kValMask; j--; }
                }
                __stcg(st, kFlagP | (excl + cnt));
            }
            gcount = a.hist[(a.shift / 8) * kRadix + d];
            g_incl = gcount;
            c_incl = cnt;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const uint64_t gv = __shfl_up_sync(0xffffffffu, g_incl, o);
                const uint32_t cv = __shfl_up_sync(0xffffffffu, c_incl, o);
                if (lane >= o) { g_incl += gv; c_incl += cv; }
            }
            if (lane == 31) { s_gw[w] = g_incl; s_cw[w] = c_incl; }
        }
        __syncthreads();
        if (d < kRadix) {
            uint64_t goff = 0;
            uint32_t coff = 0;
            for (int ww = 0; ww < w; ww++) { goff += s_gw[ww]; coff += s_cw[ww]; }
            const uint64_t g_excl = goff + g_incl - gcount;
            const uint32_t c_excl = coff + c_incl - cnt;
            s_lstart[d] = c_excl;
            s_delta[d] = g_excl + excl - c_excl;
            if (d == kRadix - 1) s_lstart[kRadix] = c_excl + cnt;
        }
        __syncthreads();
        uint64_t *s_keys = reinterpret_cast<uint64_t *>(buf);
        uint32_t *s_vals = reinterpret_cast<uint32_t *>(buf + TILE * 8);
#pragma unroll
        for (int j = 0; j < IT; j++) {
            const uint64_t i = tbase + wb + j * 32 + lane;
            if (i < a.n) {
                const uint32_t dd = (uint32_t)(key[j] >> a.shift) & 0xFF;
                const uint32_t lp = s_lstart[dd] + s_whist[w][dd] + rank[j];
                s_keys[lp] = key[j];
                s_vals[lp] = val[j];
            }
        }
        __syncthreads();
        const uint32_t nvalid = s_lstart[kRadix];
#pragma unroll 4
        for (uint32_t i = tid; i < nvalid; i += NT) {
            const uint64_t k = s_keys[i];
            const uint32_t dd = (uint32_t)(k >> a.shift) & 0xFF;
            const uint64_t gp = s_delta[dd] + i;
            if (LAST) {
                __stcs(a.t_out + gp, (uint32_t)(k & tmask));
                __stcs(a.row_out + gp, s_vals[i]);
            } else {
                __stcs(a.keys_out + gp, k);
                __stcs(a.vals_out + gp, s_vals[i]);
            }
        }
        const uint32_t nxt = s_next;
        __syncthreads();   // staging reads done before this buffer is refilled next round
        if (nxt >= ntiles) break;
        tile = nxt;
        cur ^= 1;
    }
}

template <bool FIRST, bool LAST>
static int launch_tma(const PassArgs &a, int sms, cudaStream_t st) {
    const uint32_t ntiles = (uint32_t)((a.n + kTmaTile - 1) / kTmaTile);
    const size_t smem = 2 * (size_t)kTmaTile * 12 + sizeof(uint16_t) * kRadix * (kTmaThreads / 32);
    CK(cudaFuncSetAttribute(onesweep_tma_kernel<FIRST, LAST>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                            (int)smem));
    CK(cudaFuncSetAttribute(onesweep_tma_kernel<FIRST, LAST>, cudaFuncAttributePreferredSharedMemoryCarveout, 100));
    const uint32_t grid = min(ntiles, (uint32_t)sms * 2);
    onesweep_tma_kernel<FIRST, LAST><<<grid, kTmaThreads, smem, st>>>(a, ntiles);
    return STEM_OK;
}

static int tma_sort_pass(const PassArgs &a, bool first, bool last, int sms, cudaStream_t st) {
    if (first && last) return launch_tma<true, true>(a, sms, st);
    if (first) return launch_tma<true, false>(a, sms, st);
    if (last) return launch_tma<false, true>(a, sms, st);
    return launch_tma<false, false>(a, sms, st);
}

// ---------------------------------------------------------------- reduce-then-scan pass
// (alternative to the look-back: per-tile digit counts -> one scan -> scatter)
template <int NT, int IT, bool FIRST>
__global__ void __launch_bounds__(NT) upsweep_kernel(PassArgs a, uint32_t *__restrict__ tile_hist, uint64_t ntiles) {
    constexpr int TILE = NT * IT;
    __shared__ uint32_t h[kRadix];
    for (int i = threadIdx.x; i < kRadix; i += NT) h[i] = 0;
    __syncthreads();
    const uint64_t base = (uint64_t)blockIdx.x * TILE;
#pragma unroll
    for (int j = 0; j < IT; j++) {
        const uint64_t i = base + (uint64_t)j * NT + threadIdx.x;
        if (i < a.n) {
            uint64_t k;
            if (FIRST) k = ((uint64_t)__ldg(a.kid_in + i) << a.tbits) | (uint64_t)__ldg(a.t_in + i);
            else k = __ldg(a.keys_in + i);
            atomicAdd(&h[(k >> a.shift) & 0xFF], 1u);
        }
    }
    __syncthreads();
    for (int d = threadIdx.x; d < kRadix; d += NT) tile_hist[(uint64_t)d * ntiles + blockIdx.x] = h[d];
}

template <int NT, int IT, bool FIRST, bool LAST>
__global__ void __launch_bounds__(NT, 2) downsweep_kernel(PassArgs a, const uint32_t *__restrict__ tile_off,
                                                          uint64_t ntiles) {
    constexpr int NW = NT / 32, TILE = NT * IT;
    extern __shared__ __align__(16) unsigned char s_dyn[];
    uint64_t *s_keys = reinterpret_cast<uint64_t *>(s_dyn);
    uint32_t *s_vals = reinterpret_cast<uint32_t *>(s_keys + TILE);
    uint16_t (*s_whist)[kRadix] = reinterpret_cast<uint16_t (*)[kRadix]>(s_vals + TILE);
    __shared__ uint64_t s_delta[kRadix];
    __shared__ uint32_t s_lstart[kRadix + 1];
    __shared__ uint32_t s_cw[8];
    const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
    for (int i = tid; i < NW * kRadix / 2; i += NT) reinterpret_cast<uint32_t *>(&s_whist[0][0])[i] = 0;
    __syncthreads();
    const uint32_t tile = blockIdx.x;
    const uint64_t wbase = (uint64_t)tile * TILE + (uint64_t)w * (32 * IT);
    const uint64_t tmask = (a.tbits >= 64) ? ~0ull : ((1ull << a.tbits) - 1);
    uint64_t key[IT];
    uint32_t val[IT];
#pragma unroll
    for (int j = 0; j < IT; j++) {
        const uint64_t i = wbase + (uint64_t)j * 32 + lane;
        if (i < a.n) {
            if (FIRST) {
                key[j] = ((uint64_t)__ldg(a.kid_in + i) << a.tbits) | (uint64_t)__ldg(a.t_in + i);
                val[j] = a.row_in ? __ldg(a.row_in + i) : (uint32_t)i;
            } else {
                key[j] = __ldcs(a.keys_in + i);
                val[j] = __ldcs(a.vals_in + i);
            }
        } else {
            key[j] = ~0ull;
            val[j] = 0;
        }
    }
    uint32_t rank[IT];
#pragma unroll
    for (int j = 0; j < IT; j++) {
        const uint64_t i = wbase + (uint64_t)j * 32 + lane;
        const bool valid = i < a.n;
        const uint32_t vmask = __ballot_sync(0xffffffffu, valid);
        if (valid) {
            const uint32_t d = (uint32_t)(key[j] >> a.shift) & 0xFF;
            const uint32_t peers = __match_any_sync(vmask, d);
            const uint32_t base = s_whist[w][d];
            const uint32_t below = __popc(peers & ((1u << lane) - 1));
            rank[j] = base + below;
            __syncwarp(vmask);
            if (below == 0) s_whist[w][d] = (uint16_t)(base + __popc(peers));
        }
        __syncwarp();
    }
    __syncthreads();
    const int d = tid;
    uint32_t cnt = 0, c_incl = 0;
    if (d < kRadix) {
#pragma unroll
        for (int ww = 0; ww < NW; ww++) {
            const uint32_t c = s_whist[ww][d];
            s_whist[ww][d] = (uint16_t)cnt;
            cnt += c;
        }
        c_incl = cnt;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const uint32_t cv = __shfl_up_sync(0xffffffffu, c_incl, o);
            if (lane >= o) c_incl += cv;
        }
        if (lane == 31) s_cw[w] = c_incl;
    }
    __syncthreads();
    if (d < kRadix) {
        uint32_t coff = 0;
        for (int ww = 0; ww < w; ww++) coff += s_cw[ww];
        const uint32_t c_excl = coff + c_incl - cnt;
        s_lstart[d] = c_excl;
        s_delta[d] = (uint64_t)tile_off[(uint64_t)d * ntiles + tile] - c_excl;
        if (d == kRadix - 1) s_lstart[kRadix] = c_excl + cnt;
    }
    __syncthreads();
#pragma unroll
    for (int j = 0; j < IT; j++) {
        const uint64_t i = wbase + (uint64_t)j * 32 + lane;
        if (i < a.n) {
            const uint32_t dd = (uint32_t)(key[j] >> a.shift) & 0xFF;
            const uint32_t lp = s_lstart[dd] + s_whist[w][dd] + rank[j];
            s_keys[lp] = key[j];
            s_vals[lp] = val[j];
        }
    }
    __syncthreads();
    const uint32_t nvalid = s_lstart[kRadix];
#pragma unroll 4
    for (uint32_t i = tid; i < nvalid; i += NT) {
        const uint64_t k = s_keys[i];
        const uint32_t dd = (uint32_t)(k >> a.shift) & 0xFF;
        const uint64_t gp = s_delta[dd] + i;
        if (LAST) {
            __stcs(a.t_out + gp, (uint32_t)(k & tmask));
            __stcs(a.row_out + gp, s_vals[i]);
        } else {
            __stcs(a.keys_out + gp, k);
            __stcs(a.vals_out + gp, s_vals[i]);
        }
    }
}

template <int NT, int IT, bool FIRST, bool LAST>
static int rts_pass(Ctx &c, const PassArgs &a, cudaStream_t st) {
    constexpr int TILE = NT * IT;
    const uint64_t ntiles = (a.n + TILE - 1) / TILE;
    const uint64_t cells = ntiles * kRadix;
    CKS(c.ensure(c.sort_status, c.cap_status, cells * sizeof(uint32_t) * 2));
    uint32_t *hist = (uint32_t *)c.sort_status, *off = hist + cells;
    upsweep_kernel<NT, IT, FIRST><<<(unsigned)ntiles, NT, 0, st>>>(a, hist, ntiles);
    CKS(c.ensure(c.scan_scratch, c.cap_scan, (scan_tiles(cells) + 1) * sizeof(uint64_t)));
    exclusive_scan<uint64_t>([hist] __device__(uint64_t i) -> uint64_t { return hist[i]; },
                             [off] __device__(uint64_t i, uint64_t pre, uint64_t) { off[i] = (uint32_t)pre; }, cells,
                             (uint64_t *)c.scan_scratch, &c.scalars->scan_total64, st, &c.launches);
    const size_t smem = (size_t)TILE * 12 + sizeof(uint16_t) * kRadix * (NT / 32);
    CK(cudaFuncSetAttribute(downsweep_kernel<NT, IT, FIRST, LAST>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                            (int)smem));
    CK(cudaFuncSetAttribute(downsweep_kernel<NT, IT, FIRST, LAST>, cudaFuncAttributePreferredSharedMemoryCarveout,
                            100));
    downsweep_kernel<NT, IT, FIRST, LAST><<<(unsigned)ntiles, NT, smem, st>>>(a, off, ntiles);
    c.launches += 2;
    return STEM_OK;
}

static int rts_sort_pass(Ctx &c, const PassArgs &a, bool first, bool last, cudaStream_t st) {
    if (first && last) return rts_pass<512, 8, true, true>(c, a, st);
    if (first) return rts_pass<512, 8, true, false>(c, a, st);
    if (last) return rts_pass<512, 8, false, true>(c, a, st);
    return rts_pass<512, 8, false, false>(c, a, st);
}

// ---------------------------------------------------------------- host driver
template <int NT, int IT, bool FIRST, bool LAST>
static int launch_pass(const PassArgs &a, uint64_t ntiles, bool first_hist, cudaStream_t st) {
    const size_t smem = (size_t)NT * IT * (sizeof(uint64_t) + sizeof(uint32_t)) + sizeof(uint16_t) * kRadix * (NT / 32) +
                        (FIRST && first_hist ? sizeof(uint32_t) * 7 * kRadix : 0);
    CK(cudaFuncSetAttribute(onesweep_kernel<NT, IT, FIRST, LAST>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                            (int)smem));
    CK(cudaFuncSetAttribute(onesweep_kernel<NT, IT, FIRST, LAST>, cudaFuncAttributePreferredSharedMemoryCarveout,
                            100));
    onesweep_kernel<NT, IT, FIRST, LAST><<<(unsigned)ntiles, NT, smem, st>>>(a);
    return STEM_OK;
}

template <int NT, int IT>
static int launch_pass_cfg(const PassArgs &a, bool first, bool last, bool first_hist, cudaStream_t st) {
    const uint64_t ntiles = (a.n + (uint64_t)NT * IT - 1) / ((uint64_t)NT * IT);
    if (first && last) return launch_pass<NT, IT, true, true>(a, ntiles, first_hist, st);
    if (first) return launch_pass<NT, IT, true, false>(a, ntiles, first_hist, st);
    if (last) return launch_pass<NT, IT, false, true>(a, ntiles, first_hist, st);
    return launch_pass<NT, IT, false, false>(a, ntiles, first_hist, st);
}

// tile configurations (threads, keys per thread); STEMROOT_SORT_CFG selects one for experiments
struct SortCfg { int nt, it; };
static const SortCfg kSortCfgs[] = {{256, 16}, {512, 8}, {384, 12}, {512, 12}, {512, 8}, {512, 8},
                                    {256, 8}, {128, 16}, {256, 12}};

static int sort_cfg() {
    static int cfg = -1;
    if (cfg < 0) {
        const char *e = getenv("STEMROOT_SORT_CFG");
        cfg = e ? atoi(e) : 2;
        if (cfg < 0 || cfg > 8) cfg = 2;
    }
    return cfg;
}

static int launch_sort_pass(const PassArgs &a, bool first, bool last, bool first_hist, cudaStream_t st) {
    switch (sort_cfg()) {
        case 0: return launch_pass_cfg<256, 16>(a, first, last, first_hist, st);
        case 2: return launch_pass_cfg<384, 12>(a, first, last, first_hist, st);
        case 3: return launch_pass_cfg<512, 12>(a, first, last, first_hist, st);
        case 6: return launch_pass_cfg<256, 8>(a, first, last, first_hist, st);
        case 7: return launch_pass_cfg<128, 16>(a, first, last, first_hist, st);
        case 8: return launch_pass_cfg<256, 12>(a, first, last, first_hist, st);
        default: return launch_pass_cfg<512, 8>(a, first, last, first_hist, st);
    }
}

// the pre-pass alone (kernel-id counts, range check, max t): multi-GPU histogram
int histogram_kernels(Ctx &c, const uint32_t *kid, const uint32_t *t, uint64_t n, uint32_t K) {
    cudaStream_t st = c.stream;
    CK(cudaMemsetAsync(c.hist, 0, sizeof(uint64_t) * 12 * kRadix, st));
    const int smem_kid = (K <= 40000) ? 1 : 0;
    const size_t sm_bytes = sizeof(uint32_t) * (4 * kRadix + (smem_kid ? K : 0));
    if (sm_bytes > 48 * 1024)
        CK(cudaFuncSetAttribute(prepass_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm_bytes));
    prepass_kernel<<<c.sms * 2, 256, sm_bytes, st>>>(kid, t, n, K, smem_kid, c.kid_count, c.hist + 8 * kRadix,
                                                     &c.scalars->max_t, &c.scalars->err);
    c.launches++;
    CK(cudaGetLastError());
    return STEM_OK;
}

int sort_trace(Ctx &c, const uint32_t *kid, const uint32_t *t, const uint32_t *row_in, uint64_t n, uint32_t K) {
    cudaStream_t st = c.stream;
    // pre-pass
    CK(cudaMemsetAsync(c.kid_count, 0, sizeof(uint32_t) * (K + 1), st));
    CK(cudaMemsetAsync(c.hist, 0, sizeof(uint64_t) * 12 * kRadix, st));
    CK(cudaMemsetAsync(c.scalars, 0, sizeof(DevScalars), st));
    uint64_t *hist_t = c.hist + 8 * kRadix;   // [4][256] bytes of t (pre-pass)
    const int smem_kid = (K <= 40000) ? 1 : 0;
    const size_t sm_bytes = sizeof(uint32_t) * (4 * kRadix + (smem_kid ? K : 0));
    if (sm_bytes > 48 * 1024)
        CK(cudaFuncSetAttribute(prepass_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm_bytes));
    const int blocks = c.sms * (smem_kid && K > 8192 ? 2 : 4);
    const int tk_pre = c.stage_begin("prepass");
    prepass_kernel<<<blocks, 256, sm_bytes, st>>>(kid, t, n, K, smem_kid, c.kid_count, hist_t,
                                                  &c.scalars->max_t, &c.scalars->err);
    c.launches++;
    c.stage_end(tk_pre, 8 * n);
    CK(cudaGetLastError());
    DevScalars hs;
    CK(cudaMemcpyAsync(&hs, c.scalars, sizeof(DevScalars), cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
    if (hs.err) return STEM_E_RANGE;
    int kbits = 0;
    while (kbits < 32 && ((uint64_t)1 << kbits) < (uint64_t)K) kbits++;
    int tb = 0;
    while (tb < 32 && ((uint64_t)1 << tb) <= (uint64_t)hs.max_t) tb++;
    if (tb < 8) tb = 8;
    // key = kernel_id << tbits | t.  Aligned layout (tbits a multiple of 8): every digit is a
    // byte of t or of kernel_id, all histograms come from the pre-pass.  Packed layout (tbits
    // exact) saves a pass in some traces; its later-digit histograms are built by pass 0.
    const int tb8 = (tb + 7) & ~7;
    const int passes_aligned = tb8 / 8 + (kbits + 7) / 8;
    const int passes_packed = (kbits + tb + 7) / 8;
    const bool aligned = passes_aligned <= passes_packed;
    const int tbits = aligned ? tb8 : tb;
    const int npasses = aligned ? passes_aligned : passes_packed;
    if (aligned) {
        CK(cudaMemcpyAsync(c.hist, hist_t, sizeof(uint64_t) * kRadix * (tb8 / 8), cudaMemcpyDeviceToDevice, st));
        if (kbits) {
            kid_digit_hist_kernel<<<(unsigned)((K + 255) / 256), 256, 0, st>>>(c.kid_count, K, (kbits + 7) / 8,
                                                                              c.hist + kRadix * (tb8 / 8));
            c.launches++;
        }
    } else {
        CK(cudaMemcpyAsync(c.hist, hist_t, sizeof(uint64_t) * kRadix, cudaMemcpyDeviceToDevice, st));
    }
    c.stats.key_bits = kbits + tbits;
    c.stats.sort_passes = npasses;
    c.tbits = tbits;

    const bool rts = sort_cfg() == 4;   // reduce-then-scan passes (no look-back)
    const bool tma = sort_cfg() == 5;   // persistent blocks, TMA prefetch of the next tile
    const SortCfg cfg = kSortCfgs[(rts || tma) ? 1 : sort_cfg()];
    const uint64_t ntiles = (n + (uint64_t)cfg.nt * cfg.it - 1) / ((uint64_t)cfg.nt * cfg.it);
    CKS(c.ensure(c.sort_status, c.cap_status, ntiles * kRadix * sizeof(uint64_t)));
    PassArgs a{};
    a.n = n;
    a.tbits = tbits;
    a.npasses = npasses;
    a.first_hist = aligned ? 0 : 1;
    a.hist = c.hist;
    a.hist_all = c.hist;
    a.status = (uint64_t *)c.sort_status;
    a.tile_counter = &c.scalars->tile_counter;
    uint64_t *kin = c.keys[0], *kout = c.keys[1];
    uint32_t *vin = c.vals[0], *vout = c.vals[1];
    for (int p = 0; p < npasses; p++) {
        CK(cudaMemsetAsync(a.status, 0, ntiles * kRadix * sizeof(uint64_t), st));
        CK(cudaMemsetAsync(a.tile_counter, 0, sizeof(uint32_t), st));
        a.shift = 8 * p;
        const bool first = p == 0, last = p == npasses - 1;
        a.kid_in = kid;
        a.t_in = t;
        a.row_in = row_in;
        a.keys_in = kin;
        a.vals_in = vin;
        a.keys_out = kout;
        a.vals_out = vout;
        a.t_out = c.t_sorted;
        a.row_out = c.row_sorted;
        const char *sname = (first && last) ? "sort_pass_only" : first ? "sort_pass_first"
                            : last ? "sort_pass_last" : "sort_pass_mid";
        const uint64_t sbytes = n * ((first ? 8 : 12) + (last ? 8 : 12));
        const int tk = c.stage_begin(sname);
        if (rts && (!first || aligned)) {
            CKS(rts_sort_pass(c, a, first, last, st));
        } else if (tma && (!first || aligned) &&
                   !(first && ((reinterpret_cast<uintptr_t>(kid) | reinterpret_cast<uintptr_t>(t)) & 15))) {
            CKS(tma_sort_pass(a, first, last, c.sms, st));
        } else {
            CKS(launch_sort_pass(a, first, last, !aligned, st));
        }
        c.launches++;
        c.stage_end(tk, sbytes);
        CK(cudaGetLastError());
        uint64_t *tkk = kin; kin = kout; kout = tkk;
        uint32_t *tv = vin; vin = vout; vout = tv;
    }
    // group offsets: goff = exclusive scan of kernel counts
    const uint32_t *cnt = c.kid_count;
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
