// sort.cu -- step a1 (group by kernel): stable LSD radix sort of the
// key (kernel_id << tbits | t) carrying the trace row, one-sweep style
// (Adinets & Merrill): every pass reads and writes the data once; tiles get
// their global digit offsets by decoupled look-back.
//
// Digits are RB = 8 bits wide (256 buckets) and tbits is rounded up to a
// multiple of RB, so every digit is a byte of t or of kernel_id alone: the
// pre-pass (one read of the trace) yields the histograms of every pass; the
// pass count is ceil(bits(max t)/8) + ceil(bits(K-1)/8) (6 for C5, whose
// lognormal tails reach 2^32 ns).  STEMROOT_SORT_RADIX=9 selects 9-bit digits
// (512 threads x 9 keys per tile): fewer passes on some traces, but each pass
// measured ~20% slower on B200, so bytes are the default.
#include <cstdlib>

#include "internal.h"

namespace sr {

constexpr uint64_t kFlagA = 1ull << 62, kFlagP = 2ull << 62, kValMask = (1ull << 62) - 1;
constexpr int kMaxPasses = 8;      // (24 + 32) / 8
constexpr int kTWindows = 4;       // windows of t histogrammed by the pre-pass
constexpr int kHistR = 512;        // histogram row stride (max radix)

static int radix_bits() {
    static int rb = 0;
    if (!rb) {
        const char *e = getenv("STEMROOT_SORT_RADIX");
        rb = (e && atoi(e) == 9) ? 9 : 8;
    }
    return rb;
}

// ---------------------------------------------------------------- pre-pass
// kernel-id counts (group sizes), kernel-id range check, max t, and the
// histograms of the RB-bit windows of t at bits 0, RB, 2RB, 3RB.
template <int RB>
__global__ void __launch_bounds__(256) prepass_kernel(const uint32_t *__restrict__ kid, const uint32_t *__restrict__ t,
                                                      uint64_t n, uint32_t K, int smem_kid_hist,
                                                      uint32_t *__restrict__ kid_count, uint64_t *__restrict__ hist_t,
                                                      uint32_t *__restrict__ max_t, uint32_t *__restrict__ err) {
    constexpr int R = 1 << RB;
    extern __shared__ uint32_t sh[];   // [kTWindows][R] window histograms, then [K] kernel counts
    uint32_t *h0 = sh, *hk = sh + kTWindows * R;
    for (int i = threadIdx.x; i < kTWindows * R; i += blockDim.x) h0[i] = 0;
    if (smem_kid_hist)
        for (uint32_t i = threadIdx.x; i < K; i += blockDim.x) hk[i] = 0;
    __syncthreads();
    uint32_t mx = 0, bad = 0;
    const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    const uint64_t n4 = n / 4;
    const uint4 *kid4 = reinterpret_cast<const uint4 *>(kid), *t4 = reinterpret_cast<const uint4 *>(t);
    auto one = [&](uint32_t k, uint32_t x) {
        mx = max(mx, x);
#pragma unroll
        for (int w = 0; w < kTWindows; w++) {
            const int sh_ = w * RB;
            if (sh_ < 32) atomicAdd(&h0[w * R + ((x >> sh_) & (R - 1))], 1u);
        }
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
    for (int o = 16; o; o >>= 1) {
        mx = max(mx, __shfl_xor_sync(0xffffffffu, mx, o));
        bad |= __shfl_xor_sync(0xffffffffu, bad, o);
    }
    if ((threadIdx.x & 31) == 0) {
        if (mx) atomicMax(max_t, mx);
        if (bad) atomicOr(err, 1u);
    }
    __syncthreads();
    for (int w = 0; w < kTWindows; w++)
        for (int i = threadIdx.x; i < R; i += blockDim.x)
            if (h0[w * R + i]) atomicAdd((unsigned long long *)&hist_t[w * kHistR + i], (unsigned long long)h0[w * R + i]);
    if (smem_kid_hist)
        for (uint32_t i = threadIdx.x; i < K; i += blockDim.x)
            if (hk[i]) atomicAdd(&kid_count[i], hk[i]);
}

// histograms of the kernel-id digits of the aligned key, from the kernel-id counts
__global__ void kid_digit_hist_kernel(const uint32_t *__restrict__ kid_count, uint32_t K, int rb, int ndig,
                                      uint64_t *__restrict__ hist) {
    const uint64_t g = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (g >= K || kid_count[g] == 0) return;
    for (int b = 0; b < ndig; b++)
        atomicAdd((unsigned long long *)&hist[b * kHistR + ((g >> (rb * b)) & ((1u << rb) - 1))],
                  (unsigned long long)kid_count[g]);
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
    int shift, tbits, pass;
    int ballot_rank;                    // 1: equal-digit lanes by RB ballots instead of match.any
    const uint64_t *hist;               // [pass][kHistR] global digit counts
    uint64_t *status;                   // [ntiles][R]
    uint32_t *tile_counter;
};

// One LSD pass over digit (key >> shift) & (R-1).  NT threads, IT keys per
// thread; keys loaded warp-striped (coalesced), the tile's digit counts are
// published first (flag A), keys ranked in element order by warp-level
// multi-split (match.any), global offsets found by decoupled look-back
// (thread d < R owns digit d), then keys are staged in shared memory in
// tile-sorted order and written out in digit runs (coalesced).
template <int NT, int IT, int RB, bool FIRST, bool LAST>
__global__ void __launch_bounds__(NT, (NT >= 448 ? 2 : NT >= 320 ? 3 : 4)) onesweep_kernel(PassArgs a) {
    constexpr int NW = NT / 32, TILE = NT * IT, R = 1 << RB;
    static_assert(NT >= R, "one thread per digit");
    extern __shared__ __align__(16) unsigned char s_dyn[];
    uint64_t *s_keys = reinterpret_cast<uint64_t *>(s_dyn);                           // [TILE]
    uint32_t *s_vals = reinterpret_cast<uint32_t *>(s_keys + TILE);                   // [TILE]
    uint16_t (*s_whist)[R] = reinterpret_cast<uint16_t (*)[R]>(s_vals + TILE);        // [NW][R]
    __shared__ uint64_t s_delta[R];
    __shared__ uint32_t s_lstart[R + 1];
    __shared__ uint32_t s_cnt[R];
    __shared__ uint64_t s_gw[NW];
    __shared__ uint32_t s_cw[NW];
    __shared__ uint32_t s_tile;

    const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
    if (tid == 0) s_tile = atomicAdd(a.tile_counter, 1u);
    for (int i = tid; i < NW * R / 2; i += NT) reinterpret_cast<uint32_t *>(&s_whist[0][0])[i] = 0;
    for (int i = tid; i < R; i += NT) s_cnt[i] = 0;
    __syncthreads();
    const uint32_t tile = s_tile;
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
    // the tile's digit counts, published at once so that successors' look-backs
    // do not wait for this tile's ranking
#pragma unroll
    for (int j = 0; j < IT; j++)
        if (wbase + (uint64_t)j * 32 + lane < a.n) atomicAdd(&s_cnt[(uint32_t)(key[j] >> a.shift) & (R - 1)], 1u);
    __syncthreads();
    if (tid < R) __stcg(a.status + (uint64_t)tile * R + tid, (tile == 0 ? kFlagP : kFlagA) | s_cnt[tid]);

    // warp-level multi-split ranking, in element order
    uint32_t rank[IT];
#pragma unroll
    for (int j = 0; j < IT; j++) {
        const uint64_t i = wbase + (uint64_t)j * 32 + lane;
        const bool valid = i < a.n;
        const uint32_t vmask = __ballot_sync(0xffffffffu, valid);
        if (valid) {
            const uint32_t d = (uint32_t)(key[j] >> a.shift) & (R - 1);
            uint32_t peers;
            if (a.ballot_rank) {   // lanes with an equal digit from RB ballots (no match.any)
                peers = vmask;
#pragma unroll
                for (int b = 0; b < RB; b++) {
                    const uint32_t bal = __ballot_sync(vmask, (d >> b) & 1u);
                    peers &= ((d >> b) & 1u) ? bal : ~bal;
                }
            } else {
                peers = __match_any_sync(vmask, d);
            }
            const uint32_t base = s_whist[w][d];
            const uint32_t below = __popc(peers & ((1u << lane) - 1));
            rank[j] = base + below;
            __syncwarp(vmask);
            if (below == 0) s_whist[w][d] = (uint16_t)(base + __popc(peers));
        }
        __syncwarp();
    }
    __syncthreads();

    // digit phase (threads d < R): warp offsets, look-back, global offsets
    const int d = tid;
    uint32_t cnt = 0, c_incl = 0;
    uint64_t excl = 0, gcount = 0, g_incl = 0;
    if (d < R) {
#pragma unroll
        for (int ww = 0; ww < NW; ww++) {
            const uint32_t c = s_whist[ww][d];
            s_whist[ww][d] = (uint16_t)cnt;
            cnt += c;
        }
        if (tile != 0) {
            int64_t j = (int64_t)tile - 1;
            while (true) {
                const uint64_t sv = *(volatile uint64_t *)(a.status + (uint64_t)j * R + d);
                if (sv & kFlagP) { excl += sv & kValMask; break; }
                if (sv & kFlagA) { excl += sv & kValMask; j--; }
            }
            __stcg(a.status + (uint64_t)tile * R + d, kFlagP | (excl + cnt));
        }
        gcount = a.hist[a.pass * kHistR + d];
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
    if (d < R) {
        uint64_t goff = 0;
        uint32_t coff = 0;
        for (int ww = 0; ww < w; ww++) { goff += s_gw[ww]; coff += s_cw[ww]; }
        const uint64_t g_excl = goff + g_incl - gcount;
        const uint32_t c_excl = coff + c_incl - cnt;
        s_lstart[d] = c_excl;
        s_delta[d] = g_excl + excl - c_excl;   // global position - local position
        if (d == R - 1) s_lstart[R] = c_excl + cnt;
    }
    __syncthreads();

    // scatter into shared memory in tile-sorted order, then out in digit runs
#pragma unroll
    for (int j = 0; j < IT; j++) {
        const uint64_t i = wbase + (uint64_t)j * 32 + lane;
        if (i < a.n) {
            const uint32_t dd = (uint32_t)(key[j] >> a.shift) & (R - 1);
            const uint32_t lp = s_lstart[dd] + s_whist[w][dd] + rank[j];
            s_keys[lp] = key[j];
            s_vals[lp] = val[j];
        }
    }
    __syncthreads();
    const uint32_t nvalid = s_lstart[R];
#pragma unroll 4
    for (uint32_t i = tid; i < nvalid; i += NT) {
        const uint64_t k = s_keys[i];
        const uint32_t dd = (uint32_t)(k >> a.shift) & (R - 1);
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

// ---------------------------------------------------------------- host driver
template <int NT, int IT, int RB, bool FIRST, bool LAST>
static int launch_pass(const PassArgs &a, cudaStream_t st) {
    const uint64_t ntiles = (a.n + (uint64_t)NT * IT - 1) / ((uint64_t)NT * IT);
    const size_t smem = (size_t)NT * IT * (sizeof(uint64_t) + sizeof(uint32_t)) + sizeof(uint16_t) * (NT / 32) * (1 << RB);
    CK(cudaFuncSetAttribute(onesweep_kernel<NT, IT, RB, FIRST, LAST>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                            (int)smem));
    CK(cudaFuncSetAttribute(onesweep_kernel<NT, IT, RB, FIRST, LAST>, cudaFuncAttributePreferredSharedMemoryCarveout,
                            100));
    onesweep_kernel<NT, IT, RB, FIRST, LAST><<<(unsigned)ntiles, NT, smem, st>>>(a);
    return STEM_OK;
}

template <int NT, int IT, int RB>
static int launch_pass_cfg(const PassArgs &a, bool first, bool last, cudaStream_t st) {
    if (first && last) return launch_pass<NT, IT, RB, true, true>(a, st);
    if (first) return launch_pass<NT, IT, RB, true, false>(a, st);
    if (last) return launch_pass<NT, IT, RB, false, true>(a, st);
    return launch_pass<NT, IT, RB, false, false>(a, st);
}

// tile shapes: 9-bit digits need >= 512 threads (one per digit); 8-bit keep 384 x 12
// 8-bit tile shapes (threads, keys per thread); STEMROOT_SORT_SHAPE picks one for experiments
struct Shape { int nt, it; };
static const Shape kShapes[] = {{384, 12}, {384, 10}, {320, 14}, {448, 10}, {256, 20}, {512, 9}};
static int shape_idx() {
    static int s = -1;
    if (s < 0) {
        const char *e = getenv("STEMROOT_SORT_SHAPE");
        s = e ? atoi(e) : 0;
        if (s < 0 || s > 5) s = 0;
    }
    return s;
}

static uint64_t tile_keys(int rb) {
    return rb == 9 ? 512 * 9 : (uint64_t)kShapes[shape_idx()].nt * kShapes[shape_idx()].it;
}

static int launch_sort_pass(const PassArgs &a, int rb, bool first, bool last, cudaStream_t st) {
    if (rb == 9) return launch_pass_cfg<512, 9, 9>(a, first, last, st);
    switch (shape_idx()) {
        case 1: return launch_pass_cfg<384, 10, 8>(a, first, last, st);
        case 2: return launch_pass_cfg<320, 14, 8>(a, first, last, st);
        case 3: return launch_pass_cfg<448, 10, 8>(a, first, last, st);
        case 4: return launch_pass_cfg<256, 20, 8>(a, first, last, st);
        case 5: return launch_pass_cfg<512, 9, 8>(a, first, last, st);
        default: return launch_pass_cfg<384, 12, 8>(a, first, last, st);
    }
}

template <int RB>
static int launch_prepass(Ctx &c, const uint32_t *kid, const uint32_t *t, uint64_t n, uint32_t K, uint64_t *hist_t) {
    const int smem_kid = (K <= 40000) ? 1 : 0;
    const size_t sm_bytes = sizeof(uint32_t) * (kTWindows * (1 << RB) + (smem_kid ? K : 0));
    if (sm_bytes > 48 * 1024)
        CK(cudaFuncSetAttribute(prepass_kernel<RB>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm_bytes));
    const int blocks = c.sms * (smem_kid && K > 8192 ? 2 : 4);
    prepass_kernel<RB><<<blocks, 256, sm_bytes, c.stream>>>(kid, t, n, K, smem_kid, c.kid_count, hist_t,
                                                            &c.scalars->max_t, &c.scalars->err);
    c.launches++;
    CK(cudaGetLastError());
    return STEM_OK;
}

// the pre-pass alone (kernel-id counts, range check, max t): multi-GPU histogram
int histogram_kernels(Ctx &c, const uint32_t *kid, const uint32_t *t, uint64_t n, uint32_t K) {
    CK(cudaMemsetAsync(c.hist, 0, sizeof(uint64_t) * 12 * kHistR, c.stream));
    return radix_bits() == 9 ? launch_prepass<9>(c, kid, t, n, K, c.hist + 8 * kHistR)
                             : launch_prepass<8>(c, kid, t, n, K, c.hist + 8 * kHistR);
}

int sort_trace(Ctx &c, const uint32_t *kid, const uint32_t *t, const uint32_t *row_in, uint64_t n, uint32_t K) {
    cudaStream_t st = c.stream;
    const int rb = radix_bits();
    CK(cudaMemsetAsync(c.kid_count, 0, sizeof(uint32_t) * (K + 1), st));
    CK(cudaMemsetAsync(c.scalars, 0, sizeof(DevScalars), st));
    uint64_t *hist_t = c.hist + 8 * kHistR;   // [kTWindows][kHistR] windows of t (pre-pass)
    const int tk_pre = c.stage_begin("prepass");
    CKS(histogram_kernels(c, kid, t, n, K));
    c.stage_end(tk_pre, 8 * n);
    DevScalars hs;
    CK(cudaMemcpyAsync(&hs, c.scalars, sizeof(DevScalars), cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
    if (hs.err) return STEM_E_RANGE;
    int kbits = 0;
    while (kbits < 32 && ((uint64_t)1 << kbits) < (uint64_t)K) kbits++;
    int tb = 0;
    while (tb < 32 && ((uint64_t)1 << tb) <= (uint64_t)hs.max_t) tb++;
    // key = kernel_id << tbits | t with tbits a multiple of RB: every digit is a window
    // of t (histogram from the pre-pass) or of kernel_id (from the kernel counts)
    const int tdig = tb ? (tb + rb - 1) / rb : 1;
    const int kdig = (kbits + rb - 1) / rb;
    const int tbits = tdig * rb;
    const int npasses = tdig + kdig;
    if (npasses > kMaxPasses || tdig > kTWindows) return STEM_E_RANGE;
    CK(cudaMemcpyAsync(c.hist, hist_t, sizeof(uint64_t) * kHistR * tdig, cudaMemcpyDeviceToDevice, st));
    if (kdig) {
        kid_digit_hist_kernel<<<(unsigned)((K + 255) / 256), 256, 0, st>>>(c.kid_count, K, rb, kdig,
                                                                          c.hist + kHistR * tdig);
        c.launches++;
    }
    c.stats.key_bits = kbits + tbits;
    c.stats.sort_passes = npasses;
    c.tbits = tbits;

    const uint64_t ntiles = (n + tile_keys(rb) - 1) / tile_keys(rb);
    CKS(c.ensure(c.sort_status, c.cap_status, ntiles * (1u << rb) * sizeof(uint64_t)));
    PassArgs a{};
    a.n = n;
    a.tbits = tbits;
    a.hist = c.hist;
    a.status = (uint64_t *)c.sort_status;
    a.tile_counter = &c.scalars->tile_counter;
    {
        const char *e = getenv("STEMROOT_SORT_RANK");
        a.ballot_rank = (e && e[0] == 'b') ? 1 : 0;
    }
    uint64_t *kin = c.keys[0], *kout = c.keys[1];
    uint32_t *vin = c.vals[0], *vout = c.vals[1];
    for (int p = 0; p < npasses; p++) {
        CK(cudaMemsetAsync(a.status, 0, ntiles * (1u << rb) * sizeof(uint64_t), st));
        CK(cudaMemsetAsync(a.tile_counter, 0, sizeof(uint32_t), st));
        a.shift = rb * p;
        a.pass = p;
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
        CKS(launch_sort_pass(a, rb, first, last, st));
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
