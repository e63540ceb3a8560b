// sort.cu -- step a1 (group by kernel): stable LSD radix sort of the
// packed key (kernel_id << tbits | t) carrying the trace row, one-sweep style
// (Adinets & Merrill): every pass reads and writes the data once, tiles get
// their global digit offsets by decoupled look-back.  The pre-pass validates
// kernel ids, finds max t, histograms kernel ids (group sizes) and digit 0;
// pass 0 histograms all later digits, so no extra histogram pass is needed.
#include "internal.h"

namespace sr {

constexpr int kSortThreads = 256;   // = radix: thread d owns digit d in the block phases
constexpr int kSortItems = 16;
constexpr int kSortTile = kSortThreads * kSortItems;   // 4096 keys
constexpr int kRadix = 256;
constexpr int kSortWarps = kSortThreads / 32;
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

template <bool FIRST, bool LAST>
__global__ void __launch_bounds__(kSortThreads, 3) onesweep_kernel(PassArgs a) {
    extern __shared__ __align__(16) unsigned char s_dyn[];
    uint64_t *s_keys = reinterpret_cast<uint64_t *>(s_dyn);                        // [kSortTile]
    uint32_t *s_vals = reinterpret_cast<uint32_t *>(s_keys + kSortTile);           // [kSortTile]
    uint32_t (*s_whist)[kRadix] = reinterpret_cast<uint32_t (*)[kRadix]>(s_vals + kSortTile);  // [warps][radix]
    uint32_t (*s_hlater)[kRadix] = s_whist + kSortWarps;                            // FIRST: [7][radix]
    __shared__ uint64_t s_delta[kRadix];
    __shared__ uint32_t s_lstart[kRadix + 1];
    __shared__ uint32_t s_tile;

    const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
    if (tid == 0) s_tile = atomicAdd(a.tile_counter, 1u);
    for (int i = tid; i < kSortWarps * kRadix; i += kSortThreads) (&s_whist[0][0])[i] = 0;
    if (FIRST && a.first_hist)
        for (int i = tid; i < 7 * kRadix; i += kSortThreads) (&s_hlater[0][0])[i] = 0;
    __syncthreads();
    const uint32_t tile = s_tile;
    const uint64_t tile_base = (uint64_t)tile * kSortTile;
    const uint64_t wbase = tile_base + (uint64_t)w * (32 * kSortItems);
    const uint64_t tmask = (a.tbits >= 64) ? ~0ull : ((1ull << a.tbits) - 1);

    // load (warp-striped: item j of lane l is element wbase + 32 j + l)
    uint64_t key[kSortItems];
    uint32_t val[kSortItems];
#pragma unroll
    for (int j = 0; j < kSortItems; j++) {
        const uint64_t i = wbase + (uint64_t)j * 32 + lane;
        if (i < a.n) {
            if (FIRST) {
                key[j] = ((uint64_t)__ldg(a.kid_in + i) << a.tbits) | (uint64_t)__ldg(a.t_in + i);
                val[j] = (uint32_t)i;
            } else {
                key[j] = a.keys_in[i];
                val[j] = a.vals_in[i];
            }
        } else {
            key[j] = ~0ull;
            val[j] = 0;
        }
    }
    if (FIRST && a.first_hist) {   // histograms of the later digits (each key seen exactly once here)
#pragma unroll
        for (int j = 0; j < kSortItems; j++) {
            const uint64_t i = wbase + (uint64_t)j * 32 + lane;
            if (i < a.n)
                for (int p = 1; p < a.npasses; p++) atomicAdd(&s_hlater[p - 1][(key[j] >> (8 * p)) & 0xFF], 1u);
        }
    }

    // warp-level multi-split ranking, in element order
    uint32_t rank[kSortItems];
#pragma unroll
    for (int j = 0; j < kSortItems; j++) {
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
            if (below == 0) s_whist[w][d] = base + __popc(peers);
        }
        __syncwarp();
    }
    __syncthreads();

    // per digit: exclusive offsets over warps and tile count
    const int d = tid;
    uint32_t cnt = 0;
#pragma unroll
    for (int ww = 0; ww < kSortWarps; ww++) {
        const uint32_t c = s_whist[ww][d];
        s_whist[ww][d] = cnt;
        cnt += c;
    }
    // decoupled look-back on digit d
    uint64_t *st = a.status + (uint64_t)tile * kRadix + d;
    if (tile == 0) {
        __stcg(st, kFlagP | cnt);
    } else {
        __stcg(st, kFlagA | cnt);
        uint64_t excl = 0;
        int64_t j = (int64_t)tile - 1;
        while (true) {
            const uint64_t s = *(volatile uint64_t *)(a.status + (uint64_t)j * kRadix + d);
            if (s & kFlagP) { excl += s & kValMask; break; }
            if (s & kFlagA) { excl += s & kValMask; j--; continue; }
        }
        __stcg(st, kFlagP | (excl + cnt));
        s_delta[d] = excl;  // temporarily the tile's exclusive prefix within digit d
    }
    if (tile == 0) s_delta[d] = 0;
    // global bucket base for digit d (exclusive scan of the pass histogram)
    const int pass = a.shift / 8;
    const uint64_t gcount = a.hist[pass * kRadix + d];
    // block exclusive scan over digits of (gcount) and of (cnt)
    {
        uint64_t g_incl = gcount;
        uint32_t c_incl = cnt;
        for (int o = 1; o < 32; o <<= 1) {
            const uint64_t gv = __shfl_up_sync(0xffffffffu, g_incl, o);
            const uint32_t cv = __shfl_up_sync(0xffffffffu, c_incl, o);
            if (lane >= o) { g_incl += gv; c_incl += cv; }
        }
        __shared__ uint64_t s_gw[kSortWarps];
        __shared__ uint32_t s_cw[kSortWarps];
        if (lane == 31) { s_gw[w] = g_incl; s_cw[w] = c_incl; }
        __syncthreads();
        uint64_t goff = 0;
        uint32_t coff = 0;
        for (int ww = 0; ww < w; ww++) { goff += s_gw[ww]; coff += s_cw[ww]; }
        const uint64_t g_excl = goff + g_incl - gcount;
        const uint32_t c_excl = coff + c_incl - cnt;
        s_lstart[d] = c_excl;
        s_delta[d] = g_excl + s_delta[d] - c_excl;   // global position - local position
        if (d == kRadix - 1) s_lstart[kRadix] = c_excl + cnt;
    }
    if (FIRST && a.first_hist) {
        for (int p = 1; p < a.npasses; p++) {
            const uint32_t h = s_hlater[p - 1][d];
            if (h) atomicAdd((unsigned long long *)&a.hist_all[p * kRadix + d], (unsigned long long)h);
        }
    }
    __syncthreads();

    // scatter into shared memory in tile-sorted order
#pragma unroll
    for (int j = 0; j < kSortItems; j++) {
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
    for (uint32_t i = tid; i < nvalid; i += kSortThreads) {
        const uint64_t k = s_keys[i];
        const uint32_t dd = (uint32_t)(k >> a.shift) & 0xFF;
        const uint64_t gp = s_delta[dd] + i;
        if (LAST) {
            a.t_out[gp] = (uint32_t)(k & tmask);
            a.row_out[gp] = s_vals[i];
        } else {
            a.keys_out[gp] = k;
            a.vals_out[gp] = s_vals[i];
        }
    }
}

// ---------------------------------------------------------------- host driver
template <bool FIRST, bool LAST>
static int launch_pass(const PassArgs &a, uint64_t ntiles, size_t smem, cudaStream_t st) {
    CK(cudaFuncSetAttribute(onesweep_kernel<FIRST, LAST>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    CK(cudaFuncSetAttribute(onesweep_kernel<FIRST, LAST>, cudaFuncAttributePreferredSharedMemoryCarveout, 100));
    onesweep_kernel<FIRST, LAST><<<(unsigned)ntiles, kSortThreads, smem, st>>>(a);
    return STEM_OK;
}

int sort_trace(Ctx &c, const uint32_t *kid, const uint32_t *t, uint64_t n, uint32_t K) {
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

    const uint64_t ntiles = (n + kSortTile - 1) / kSortTile;
    c.ensure(c.sort_status, c.cap_status, ntiles * kRadix * sizeof(uint64_t));
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
        a.keys_in = kin;
        a.vals_in = vin;
        a.keys_out = kout;
        a.vals_out = vout;
        a.t_out = c.t_sorted;
        a.row_out = c.row_sorted;
        const size_t smem = kSortTile * (sizeof(uint64_t) + sizeof(uint32_t)) +
                            sizeof(uint32_t) * kRadix * (kSortWarps + (first && !aligned ? 7 : 0));
        const char *sname = (first && last) ? "sort_pass_only" : first ? "sort_pass_first"
                            : last ? "sort_pass_last" : "sort_pass_mid";
        const uint64_t sbytes = n * ((first ? 8 : 12) + (last ? 8 : 12));
        const int tk = c.stage_begin(sname);
        int rc;
        if (first && last) rc = launch_pass<true, true>(a, ntiles, smem, st);
        else if (first) rc = launch_pass<true, false>(a, ntiles, smem, st);
        else if (last) rc = launch_pass<false, true>(a, ntiles, smem, st);
        else rc = launch_pass<false, false>(a, ntiles, smem, st);
        CKS(rc);
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
