// metric.cu -- step a8, option metric_bounds (R28): the true total
// of every metric column and the predicted relative error of its estimate,
// Eq. 5 with the metric in place of the execution time (the
// metrics are extrapolated like time):
//   true_c  = sum over all rows of metric_c
//   V_ic    = n_i^2 sigma_ic^2 = n_i * sum_{rows j of leaf i} (x_j - xbar_ic)^2,
//             xbar_ic = (sum_j x_j) / n_i           (population variance, R3)
//   bound_c = z sqrt(sum_i V_ic / m_i) / |true_c|
// The rows are read in TRACE order (coalesced metric columns): a leaf is the
// set of rows of one kernel with t in [lo_ns, hi_ns] (a cut never separates
// equal times), so the leaf of a row is a binary search of its t among the
// kernel's leaf lower bounds.  Two passes (sums, then squared deviations from
// the leaf mean) accumulate per-leaf fp64 sums with warp-aggregated atomics;
// the column totals use deterministic per-warp / per-block partials.
#include <cstdlib>

#include "internal.h"

namespace sr {

constexpr int kMbThreads = 256;
constexpr int kMbWarps = kMbThreads / 32;

struct MbTable {
    const uint32_t *first;   // [K + 1] first leaf of kernel k (leaves sorted by (kernel, lo))
    const uint32_t *lo_ns;   // [L] smallest t of each leaf
};

__device__ __forceinline__ uint32_t mb_leaf(const MbTable &tb, uint32_t k, uint32_t tv) {
    const uint32_t a = tb.first[k], b = tb.first[k + 1];
    return a + (uint32_t)upper_bound(tb.lo_ns + a, (uint64_t)(b - a), tv) - 1;
}

// every lane gets the sum of v over the lanes of its group `peers` (ascending lane order)
__device__ __forceinline__ double group_sum(double v, uint32_t peers) {
    double s = 0.0;
#pragma unroll
    for (int j = 0; j < 32; j++) {
        const double x = __shfl_sync(0xffffffffu, v, j);
        if ((peers >> j) & 1u) s = __dadd_rn(s, x);
    }
    return s;
}

// first[k] = first leaf of kernel k = lower_bound(leaf_kid, k), k in [0, K]
__global__ void mb_first_kernel(const uint32_t *leaf_kid, uint64_t L, uint32_t K, uint32_t *first) {
    const uint64_t k = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (k <= K) first[k] = (uint32_t)lower_bound(leaf_kid, L, (uint32_t)k);
}

// single GPU: the table columns from this plan's leaves
__global__ void mb_local_table_kernel(const uint32_t *leaf_lo, const uint32_t *t_sorted, uint64_t L, uint64_t n,
                                      uint32_t *lo_ns, uint64_t *ln) {
    const uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= L) return;
    const uint32_t lo = leaf_lo[i], hi = i + 1 < L ? leaf_lo[i + 1] : (uint32_t)n;
    lo_ns[i] = t_sorted[lo];
    ln[i] = hi - lo;
}

// pass 1: per-leaf sums of x (atomics), leaf of every row, column partials
__global__ void __launch_bounds__(kMbThreads) mb_sum_kernel(MbTable tb, const uint32_t *__restrict__ kid,
                                                           const uint32_t *__restrict__ t,
                                                           const double *__restrict__ met, uint64_t n, uint32_t nm,
                                                           uint32_t *__restrict__ leaf_of, double *acc,
                                                           double *__restrict__ part) {
    __shared__ double s_w[kMbWarps][64];
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    for (uint32_t c = lane; c < nm; c += 32) s_w[w][c] = 0.0;
    __syncwarp();
    const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    for (uint64_t r0 = (uint64_t)blockIdx.x * blockDim.x + ((uint64_t)w << 5); r0 < n; r0 += stride) {
        const uint64_t r = r0 + lane;
        const bool in = r < n;
        uint32_t leaf = 0xFFFFFFFFu;
        if (in) {
            leaf = mb_leaf(tb, kid[r], t[r]);
            leaf_of[r] = leaf;
        }
        const uint32_t peers = __match_any_sync(0xffffffffu, leaf);
        const bool lead = in && (__ffs(peers) - 1) == lane;
        const bool dup = __any_sync(0xffffffffu, __popc(peers) > 1);
        for (uint32_t c = 0; c < nm; c++) {
            const double x = in ? __ldcs(met + (uint64_t)c * n + r) : 0.0;
            const double s = dup ? group_sum(x, peers) : x;
            if (lead) atomicAdd(acc + (uint64_t)leaf * nm + c, s);
            double tsum = x;
#pragma unroll
            for (int o = 16; o; o >>= 1) tsum = __dadd_rn(tsum, __shfl_xor_sync(0xffffffffu, tsum, o));
            if (lane == 0) s_w[w][c] = __dadd_rn(s_w[w][c], tsum);
        }
    }
    __syncthreads();
    for (uint32_t c = threadIdx.x; c < nm; c += blockDim.x) {
        double s = 0.0;
        for (int k = 0; k < kMbWarps; k++) s = __dadd_rn(s, s_w[k][c]);
        part[(uint64_t)blockIdx.x * nm + c] = s;
    }
}

// xbar_ic = (sum x) / n_i, in place
__global__ void mb_mean_kernel(double *acc, const uint64_t *ln, uint64_t L, uint32_t nm) {
    const uint64_t x = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (x >= L * nm) return;
    acc[x] = __ddiv_rn(acc[x], rn64(ln[x / nm]));
}

// pass 2: per-leaf sums of (x - xbar)^2
__global__ void __launch_bounds__(kMbThreads) mb_dev_kernel(const uint32_t *__restrict__ leaf_of,
                                                           const double *__restrict__ met, uint64_t n, uint32_t nm,
                                                           const double *__restrict__ xbar, double *acc2) {
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    for (uint64_t r0 = (uint64_t)blockIdx.x * blockDim.x + ((uint64_t)w << 5); r0 < n; r0 += stride) {
        const uint64_t r = r0 + lane;
        const bool in = r < n;
        const uint32_t leaf = in ? __ldcs(leaf_of + r) : 0xFFFFFFFFu;
        const uint32_t peers = __match_any_sync(0xffffffffu, leaf);
        const bool lead = in && (__ffs(peers) - 1) == lane;
        const bool dup = __any_sync(0xffffffffu, __popc(peers) > 1);
        for (uint32_t c = 0; c < nm; c++) {
            double v = 0.0;
            if (in) {
                const double d = __dsub_rn(__ldcs(met + (uint64_t)c * n + r), xbar[(uint64_t)leaf * nm + c]);
                v = __dmul_rn(d, d);
            }
            const double s = dup ? group_sum(v, peers) : v;
            if (lead) atomicAdd(acc2 + (uint64_t)leaf * nm + c, s);
        }
    }
}

// per-block partials of sum_i (n_i * W_ic) / m_i (deterministic block order)
__global__ void __launch_bounds__(kMbThreads) mb_var_kernel(const double *__restrict__ acc2,
                                                           const uint64_t *__restrict__ ln,
                                                           const uint64_t *__restrict__ lm, uint64_t L, uint32_t nm,
                                                           double *__restrict__ part) {
    __shared__ double sm[kMbWarps];
    const uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    for (uint32_t c = 0; c < nm; c++) {
        double v = 0.0;
        if (i < L) v = __ddiv_rn(__dmul_rn(rn64(ln[i]), acc2[i * nm + c]), rn64(lm[i]));
#pragma unroll
        for (int o = 16; o; o >>= 1) v = __dadd_rn(v, __shfl_xor_sync(0xffffffffu, v, o));
        __syncthreads();
        if ((threadIdx.x & 31) == 0) sm[threadIdx.x >> 5] = v;
        __syncthreads();
        if (threadIdx.x == 0) {
            double r = 0.0;
            for (int k = 0; k < kMbWarps; k++) r = __dadd_rn(r, sm[k]);
            part[(uint64_t)blockIdx.x * nm + c] = r;
        }
    }
}

// column sums of [blocks][cols] partials in block order
__global__ void mb_cols_kernel(const double *part, uint64_t blocks, uint32_t cols, double *out) {
    const uint32_t c = blockIdx.x * blockDim.x + threadIdx.x;
    if (c >= cols) return;
    double r = 0.0;
    for (uint64_t b = 0; b < blocks; b++) r = __dadd_rn(r, part[b * cols + c]);
    out[c] = r;
}

__global__ void mb_final_kernel(const double *tru, const double *var, uint32_t nm, double z, double *bound) {
    const uint32_t c = threadIdx.x;
    if (c >= nm) return;
    const double tc = fabs(tru[c]);
    bound[c] = tc > 0.0 ? __ddiv_rn(__dmul_rn(z, __dsqrt_rn(var[c])), tc)
                        : (var[c] > 0.0 ? __longlong_as_double(0x7FF0000000000000ll) : 0.0);
}

// The table (first, lo_ns, n, m over L leaves of K kernels) must be in
// c.mb_first / c.mb_lo / c.mb_n / c.mb_m.  Rows: kid, t, met of n rows (this
// rank's home rows in multi-GPU).  Results into host true_out / bound_out.
static int metric_bounds_table_run(Ctx &c, uint64_t L, const uint32_t *kid, const uint32_t *t, const double *met,
                                   uint64_t n, uint32_t nm, double z, double *true_out, double *bound_out) {
    cudaStream_t st = c.stream;
    const uint64_t cells = L * nm;
    const unsigned grid = (unsigned)max((uint64_t)1, min((n + kMbThreads - 1) / kMbThreads, (uint64_t)c.sms * 8));
    const uint64_t vblocks = (L + kMbThreads - 1) / kMbThreads;
    CKS(dist_checkpoint(c, [&]() -> int {
        CKS(c.ensure(c.mb_acc, c.cap_mb_acc, sizeof(double) * (2 * cells + 1)));
        CKS(c.ensure(c.mb_leaf_of, c.cap_mb_leaf_of, sizeof(uint32_t) * (n + 1)));
        CKS(c.ensure(c.mb_part, c.cap_mb_part, sizeof(double) * (((uint64_t)grid + vblocks) * nm + 4 * 64)));
        return STEM_OK;
    }()));
    double *acc1 = c.mb_acc, *acc2 = c.mb_acc + cells;
    double *partA = c.mb_part, *partV = partA + (uint64_t)grid * nm, *red = partV + vblocks * nm;
    double *tru = red, *var = red + 64, *bnd = red + 128;
    const MbTable tb{c.mb_first, c.mb_lo};
    CKS(dist_checkpoint(c, [&]() -> int {
        CK(cudaMemsetAsync(c.mb_acc, 0, sizeof(double) * 2 * cells, st));
        if (n) {
            mb_sum_kernel<<<grid, kMbThreads, 0, st>>>(tb, kid, t, met, n, nm, c.mb_leaf_of, acc1, partA);
            mb_cols_kernel<<<1, 64, 0, st>>>(partA, grid, nm, tru);
            c.launches += 2;
        } else {
            CK(cudaMemsetAsync(tru, 0, sizeof(double) * nm, st));
        }
        CK(cudaGetLastError());
        return STEM_OK;
    }()));
    if (c.comm) {
        CKS(dist_allreduce_f64(c, acc1, cells));
        CKS(dist_allreduce_f64(c, tru, nm));
    }
    CKS(dist_checkpoint(c, [&]() -> int {
        if (cells) {
            mb_mean_kernel<<<(unsigned)((cells + 255) / 256), 256, 0, st>>>(acc1, c.mb_n, L, nm);
            c.launches++;
        }
        if (n) {
            mb_dev_kernel<<<grid, kMbThreads, 0, st>>>(c.mb_leaf_of, met, n, nm, acc1, acc2);
            c.launches++;
        }
        CK(cudaGetLastError());
        return STEM_OK;
    }()));
    if (c.comm) CKS(dist_allreduce_f64(c, acc2, cells));
    if (L) {
        mb_var_kernel<<<(unsigned)vblocks, kMbThreads, 0, st>>>(acc2, c.mb_n, c.mb_m, L, nm, partV);
        mb_cols_kernel<<<1, 64, 0, st>>>(partV, vblocks, nm, var);
        c.launches += 2;
    } else {
        CK(cudaMemsetAsync(var, 0, sizeof(double) * nm, st));
    }
    mb_final_kernel<<<1, 64, 0, st>>>(tru, var, nm, z, bnd);
    c.launches++;
    CK(cudaGetLastError());
    CK(cudaMemcpyAsync(true_out, tru, sizeof(double) * nm, cudaMemcpyDeviceToHost, st));
    CK(cudaMemcpyAsync(bound_out, bnd, sizeof(double) * nm, cudaMemcpyDeviceToHost, st));
    CKS(sync_stream(c));
    return STEM_OK;
}

// ---------------------------------------------------------------- sorted-order path (single GPU)
// When every sorted position's trace row is known (row payload, or a packed
// key whose low bits hold the whole row), the rows are walked in SORTED order:
// a leaf is then a contiguous run, so sums need no per-row atomics -- each
// warp walks a segment of kMbSeg positions, reduces runs of equal leaf with a
// segmented warp scan and carries the open run across its iterations; only a
// run's end (a leaf boundary, or the segment's end) is added atomically.  The
// metric values are gathered by row (random 8-byte reads).
constexpr int kMbSeg = 2048;   // sorted positions per warp

struct MbSorted {
    const uint32_t *row;        // row_sorted: the trace row of each sorted position
    const uint32_t *flags;      // leaf-start bitmap (bit p: a leaf starts at sorted position p)
    const uint32_t *leaf_lo;    // [L] leaf starts
    uint64_t L, n;
    const double *met;          // [nm][n] trace order
    uint32_t nm;
    const double *mean;         // pass 2: [L][nm] leaf means, NULL in pass 1
    double *acc;                // [L][nm]
    double *part;               // pass 1: [warps][nm] column partials (deterministic)
};

template <bool DEV>
__global__ void __launch_bounds__(kMbThreads) mb_sorted_kernel(MbSorted a) {
    __shared__ double s_carry[kMbWarps][64];
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    const uint64_t gw = ((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const uint64_t s0 = gw * kMbSeg;
    if (s0 >= a.n) return;
    const uint64_t s1 = min(a.n, s0 + kMbSeg);
    // leaf of the segment's first position (the last leaf start <= s0)
    uint64_t base_leaf = upper_bound(a.leaf_lo, a.L, (uint32_t)s0) - 1;
    const uint64_t nwords = (a.n + 31) / 32;
    uint64_t carry_leaf = ~0ull;
    for (uint32_t c = lane; c < a.nm; c += 32) s_carry[w][c] = 0.0;
    double colsum = 0.0;   // pass 1: lane c's column total over the segment (c < 32), in position order
    __syncwarp();
    for (uint64_t p0 = s0; p0 < s1; p0 += 32) {
        const uint64_t pos = p0 + lane;
        const bool in = pos < s1;
        // leaf starts at positions p0 .. p0 + 63 (bit i = position p0 + i)
        const uint64_t w0 = p0 >> 5;
        const uint64_t bits = ((uint64_t)(w0 + 1 < nwords ? a.flags[w0 + 1] : 0u) << 32 | a.flags[w0]) >> (p0 & 31);
        const uint64_t upto = bits & ((2ull << lane) - 1);
        const uint64_t leaf = base_leaf + __popcll(upto & ~1ull);   // + starts in (p0, pos]
        const uint32_t head = __ballot_sync(0xffffffffu, in && (lane == 0 || ((bits >> lane) & 1ull)));
        const uint32_t inm = __ballot_sync(0xffffffffu, in);
        const int last_in = 31 - __clz(inm);
        const int seg = 31 - __clz(head & (0xFFFFFFFFu >> (31 - lane)));   // first lane of my run
        const bool tail = in && (lane == last_in || ((head >> (lane + 1)) & 1u));
        const uint64_t leaf_first = base_leaf;
        const bool last_iter = p0 + 32 >= s1;
        const uint32_t r = in ? a.row[pos] : 0u;
        constexpr int kG = 4;   // metric columns whose gathers are in flight together
        for (uint32_t c0 = 0; c0 < a.nm; c0 += kG) {
          double xs[kG];
#pragma unroll
          for (int u = 0; u < kG; u++)
              xs[u] = (in && c0 + u < a.nm) ? __ldg(a.met + (uint64_t)(c0 + u) * a.n + r) : 0.0;
#pragma unroll 1
          for (int u = 0; u < kG && c0 + u < a.nm; u++) {
            const uint32_t c = c0 + u;
            double x = u == 0 ? xs[0] : u == 1 ? xs[1] : u == 2 ? xs[2] : xs[3];
            if (!DEV && c < 32) {   // column total (pass 1), deterministic butterfly then in order
                double tsum = x;
#pragma unroll
                for (int o = 16; o; o >>= 1) tsum = __dadd_rn(tsum, __shfl_xor_sync(0xffffffffu, tsum, o));
                if (lane == (int)c) colsum = __dadd_rn(colsum, tsum);
            }
            if (DEV && in) {
                const double d = __dsub_rn(x, a.mean[leaf * a.nm + c]);
                x = __dmul_rn(d, d);
            }
            // segmented inclusive scan over runs of equal leaf
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const double u = __shfl_up_sync(0xffffffffu, x, o);
                if (lane - o >= seg) x = __dadd_rn(x, u);
            }
            const double carry = s_carry[w][c];
            __syncwarp();
            // the open run of the previous iteration ended at its last position
            if (lane == 0 && carry_leaf != ~0ull && carry_leaf != leaf_first)
                atomicAdd(a.acc + carry_leaf * a.nm + c, carry);
            if (tail) {
                double v = x;
                if (seg == 0 && leaf == carry_leaf) v = __dadd_rn(v, carry);   // the open run continues
                if (lane == last_in && !last_iter) s_carry[w][c] = v;          // still open
                else atomicAdd(a.acc + leaf * a.nm + c, v);
            }
            __syncwarp();
          }
        }
        carry_leaf = __shfl_sync(0xffffffffu, leaf, last_in);
        base_leaf += __popcll((bits >> 1) & 0xFFFFFFFFull);   // leaf of position p0 + 32
    }
    if (!DEV) {   // column partials of this warp: lane c holds column c (c < 32), others by a second sweep
        for (uint32_t c = lane; c < a.nm && c < 32; c += 32) a.part[gw * a.nm + c] = colsum;
    }
}

// columns 32..63 of pass 1's totals (rare: more than 32 metrics), per warp in position order
__global__ void __launch_bounds__(kMbThreads) mb_sorted_cols_hi_kernel(MbSorted a) {
    const int lane = threadIdx.x & 31;
    const uint64_t gw = ((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const uint64_t s0 = gw * kMbSeg;
    if (s0 >= a.n) return;
    const uint64_t s1 = min(a.n, s0 + kMbSeg);
    for (uint32_t c = 32; c < a.nm; c++) {
        double colsum = 0.0;
        for (uint64_t p0 = s0; p0 < s1; p0 += 32) {
            const uint64_t pos = p0 + lane;
            double x = pos < s1 ? __ldg(a.met + (uint64_t)c * a.n + a.row[pos]) : 0.0;
#pragma unroll
            for (int o = 16; o; o >>= 1) x = __dadd_rn(x, __shfl_xor_sync(0xffffffffu, x, o));
            colsum = __dadd_rn(colsum, x);
        }
        if (lane == 0) a.part[gw * a.nm + c] = colsum;
    }
}

static int metric_bounds_sorted(Ctx &c, uint64_t L, uint64_t n, const double *met, uint32_t nm, double z) {
    cudaStream_t st = c.stream;
    const uint64_t cells = L * nm;
    const uint64_t warps = (n + kMbSeg - 1) / kMbSeg;
    const unsigned grid = (unsigned)((warps + kMbWarps - 1) / kMbWarps);
    const uint64_t vblocks = (L + kMbThreads - 1) / kMbThreads;
    CKS(c.ensure(c.mb_acc, c.cap_mb_acc, sizeof(double) * (2 * cells + 1)));
    CKS(c.ensure(c.mb_part, c.cap_mb_part, sizeof(double) * ((warps + vblocks) * nm + 4 * 64)));
    double *acc1 = c.mb_acc, *acc2 = c.mb_acc + cells;
    double *partA = c.mb_part, *partV = partA + warps * nm, *red = partV + vblocks * nm;
    double *tru = red, *var = red + 64, *bnd = red + 128;
    CK(cudaMemsetAsync(c.mb_acc, 0, sizeof(double) * 2 * cells, st));
    MbSorted a{c.row_sorted, c.flags, c.leaf_lo, L, n, met, nm, nullptr, acc1, partA};
    if (n) {
        mb_sorted_kernel<false><<<grid, kMbThreads, 0, st>>>(a);
        if (nm > 32) mb_sorted_cols_hi_kernel<<<grid, kMbThreads, 0, st>>>(a);
        mb_cols_kernel<<<1, 64, 0, st>>>(partA, warps, nm, tru);
        c.launches += nm > 32 ? 3 : 2;
    } else {
        CK(cudaMemsetAsync(tru, 0, sizeof(double) * nm, st));
    }
    if (cells) {
        mb_mean_kernel<<<(unsigned)((cells + 255) / 256), 256, 0, st>>>(acc1, c.mb_n, L, nm);
        c.launches++;
    }
    if (n) {
        MbSorted b{c.row_sorted, c.flags, c.leaf_lo, L, n, met, nm, acc1, acc2, nullptr};
        mb_sorted_kernel<true><<<grid, kMbThreads, 0, st>>>(b);
        c.launches++;
    }
    if (L) {
        mb_var_kernel<<<(unsigned)vblocks, kMbThreads, 0, st>>>(acc2, c.mb_n, c.mb_m, L, nm, partV);
        mb_cols_kernel<<<1, 64, 0, st>>>(partV, vblocks, nm, var);
        c.launches += 2;
    } else {
        CK(cudaMemsetAsync(var, 0, sizeof(double) * nm, st));
    }
    mb_final_kernel<<<1, 64, 0, st>>>(tru, var, nm, z, bnd);
    c.launches++;
    CK(cudaGetLastError());
    CK(cudaMemcpyAsync(c.host_true_metric, tru, sizeof(double) * nm, cudaMemcpyDeviceToHost, st));
    CK(cudaMemcpyAsync(c.host_bound_metric, bnd, sizeof(double) * nm, cudaMemcpyDeviceToHost, st));
    CKS(sync_stream(c));
    return STEM_OK;
}

// single GPU: the plan's own leaves are the table
int metric_bounds_local(Ctx &c, uint64_t L, uint32_t K, uint64_t n_sorted, const uint32_t *kid, const uint32_t *t,
                        const double *met, uint64_t n_trace, uint32_t nm, double z) {
    cudaStream_t st = c.stream;
    CKS(c.ensure(c.mb_first, c.cap_mb_first, sizeof(uint32_t) * ((uint64_t)K + 2)));
    CKS(c.ensure(c.mb_lo, c.cap_mb_lo, sizeof(uint32_t) * (L + 1)));
    CKS(c.ensure(c.mb_n, c.cap_mb_n, sizeof(uint64_t) * (L + 1)));
    mb_first_kernel<<<(unsigned)((K + 256) / 256), 256, 0, st>>>(c.leaf_kid, L, K, c.mb_first);
    if (L) mb_local_table_kernel<<<(unsigned)((L + 255) / 256), 256, 0, st>>>(c.leaf_lo, c.t_sorted, L, n_sorted, c.mb_lo,
                                                                                c.mb_n);
    c.launches += 2;
    c.mb_m = c.leaf_m;
    // every sorted position's row known (payload, or packed low bits = the whole row): sorted order
    if ((c.pack_h <= 1 && !c.sort_row_in) && !(getenv("STEMROOT_MB_TRACE_ORDER")))
        return metric_bounds_sorted(c, L, n_sorted, met, nm, z);
    return metric_bounds_table_run(c, L, kid, t, met, n_trace, nm, z, c.host_true_metric, c.host_bound_metric);
}

// multi-GPU: every rank's leaves gathered into one table (kernel ranges ascend
// with the rank, so the concatenation is in (kernel, lo) order)
struct MbRec {
    uint32_t kid, lo_ns;
    uint64_t n, m;
};

__global__ void mb_pack_kernel(const uint32_t *leaf_lo, const uint32_t *leaf_kid, const uint32_t *t_sorted,
                               const uint64_t *leaf_m, uint64_t L, uint64_t n, uint32_t kid_base, MbRec *out) {
    const uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= L) return;
    const uint32_t lo = leaf_lo[i], hi = i + 1 < L ? leaf_lo[i + 1] : (uint32_t)n;
    out[i] = MbRec{kid_base + leaf_kid[i], t_sorted[lo], (uint64_t)(hi - lo), leaf_m[i]};
}

__global__ void mb_unpack_kernel(const MbRec *in, uint64_t L, uint32_t *kid, uint32_t *lo_ns, uint64_t *ln,
                                 uint64_t *lm) {
    const uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= L) return;
    const MbRec r = in[i];
    kid[i] = r.kid;
    lo_ns[i] = r.lo_ns;
    ln[i] = r.n;
    lm[i] = r.m;
}

int metric_bounds_dist(Ctx &c, uint64_t L_local, uint64_t n_sorted, uint32_t K_global, const uint32_t *kid,
                       const uint32_t *t, const double *met, uint64_t n_home, uint32_t nm, double z) {
    cudaStream_t st = c.stream;
    const int W = comm_world(c.comm), me = comm_rank(c.comm);
    std::vector<uint64_t> all((size_t)W);
    CKS(comm_allgather_host(c, &L_local, 1, all.data()));
    uint64_t Lg = 0;
    std::vector<uint64_t> scnt(W, L_local), sdsp(W, 0), rcnt(W), rdsp(W);
    for (int r = 0; r < W; r++) {
        rcnt[r] = all[r];
        rdsp[r] = Lg;
        Lg += all[r];
    }
    (void)me;
    MbRec *mine = nullptr, *gathered = nullptr;
    CKS(dist_checkpoint(c, [&]() -> int {
        CKS(c.ensure(c.mb_rec, c.cap_mb_rec, sizeof(MbRec) * (L_local + Lg + 2)));
        mine = (MbRec *)c.mb_rec;
        gathered = mine + L_local + 1;
        if (L_local) {
            mb_pack_kernel<<<(unsigned)((L_local + 255) / 256), 256, 0, st>>>(
                c.leaf_lo, c.leaf_kid, c.t_sorted, c.leaf_m, L_local, n_sorted, c.kid_base, mine);
            c.launches++;
        }
        CK(cudaGetLastError());
        return STEM_OK;
    }()));
    CKS(comm_alltoallv(c, mine, scnt.data(), sdsp.data(), gathered, rcnt.data(), rdsp.data(), sizeof(MbRec)));
    CKS(dist_checkpoint(c, [&]() -> int {
        CKS(c.ensure(c.mb_first, c.cap_mb_first, sizeof(uint32_t) * ((uint64_t)K_global + 2)));
        CKS(c.ensure(c.mb_lo, c.cap_mb_lo, sizeof(uint32_t) * (Lg + 1)));
        CKS(c.ensure(c.mb_n, c.cap_mb_n, sizeof(uint64_t) * (Lg + 1)));
        CKS(c.ensure(c.mb_gm, c.cap_mb_gm, sizeof(uint64_t) * (Lg + 1)));
        CKS(c.ensure(c.mb_gkid, c.cap_mb_gkid, sizeof(uint32_t) * (Lg + 1)));
        if (Lg) {
            mb_unpack_kernel<<<(unsigned)((Lg + 255) / 256), 256, 0, st>>>(gathered, Lg, c.mb_gkid, c.mb_lo, c.mb_n,
                                                                           c.mb_gm);
            c.launches++;
        }
        mb_first_kernel<<<(unsigned)((K_global + 256) / 256), 256, 0, st>>>(c.mb_gkid, Lg, K_global, c.mb_first);
        c.launches++;
        c.mb_m = c.mb_gm;
        CK(cudaGetLastError());
        return STEM_OK;
    }()));
    return metric_bounds_table_run(c, Lg, kid, t, met, n_home, nm, z, c.host_true_metric, c.host_bound_metric);
}

}  // namespace sr
