// root.cu -- steps a2-a4: exact prefix moments of the grouped times and the
// level-synchronous ROOT clustering (§3.4, Fig. 6).
//
// Every level processes the whole frontier (all kernels' active clusters at
// once) as one segmented operation over the concatenated active rows:
//   split_kernel   tiles of 2048 active rows; each candidate cut k of a
//                  cluster [lo,hi) is scored exactly from P1 (D = n S_L - S k,
//                  score D^2/(k(n-k)), R5); thread-, then block-level segmented
//                  argmax; clusters inside a tile finish here.
//   fixup_kernel   one warp per cluster spanning several tiles: argmax of the
//                  per-tile partials.
//   decide_kernel  Eq. 7 vs Eq. 8 per cluster (R6-R9) in the fixed fp64 order.
//   scan + apply   compacts the non-trivial children into the next frontier.
#include "internal.h"

namespace sr {

constexpr int kSplitThreads = 256;
constexpr int kSplitItems = 8;
constexpr uint64_t kSplitTile = (uint64_t)kSplitThreads * kSplitItems;
constexpr uint32_t kNone = 0xFFFFFFFFu;

struct SQ {
    uint64_t s;
    u128 q;
};
__host__ __device__ __forceinline__ SQ operator+(const SQ &a, const SQ &b) { return SQ{a.s + b.s, a.q + b.q}; }
__host__ __device__ __forceinline__ SQ operator-(const SQ &a, const SQ &b) { return SQ{a.s - b.s, a.q - b.q}; }

// ---------------------------------------------------------------- a2: P1, P2
int prefix_moments(Ctx &c, uint64_t n) {
    const uint32_t *t = c.t_sorted;
    uint64_t *P1 = c.P1;
    u128 *P2 = c.P2;
    CKS(c.ensure(c.scan_scratch, c.cap_scan, (scan_tiles(n + 1) + 1) * sizeof(SQ)));
    const int tk = c.stage_begin("prefix_moments");
    exclusive_scan<SQ>(
        [t, n] __device__(uint64_t i) -> SQ {
            if (i >= n) return SQ{0, 0};
            const uint64_t x = t[i];
            return SQ{x, (u128)(x * x)};
        },
        [P1, P2] __device__(uint64_t i, SQ pre, SQ) {
            P1[i] = pre.s;
            P2[i] = pre.q;
        },
        n + 1, (SQ *)c.scan_scratch, (SQ *)c.scalars->wide_total,
        c.stream, &c.launches);
    c.stage_end(tk, 4 * n + 24 * (n + 1));
    CK(cudaGetLastError());
    return STEM_OK;
}

// ---------------------------------------------------------------- a3: split
struct Part {
    Cand cand;
    uint32_t c;
};

__device__ __forceinline__ bool nontrivial(const uint32_t *t, uint32_t lo, uint32_t hi) {
    return hi - lo >= 2 && t[lo] != t[hi - 1];
}

__global__ void __launch_bounds__(kSplitThreads)
split_kernel(const uint32_t *__restrict__ f_lo, const uint32_t *__restrict__ f_hi, const uint32_t *__restrict__ aoff,
             uint32_t C, uint64_t A, const uint64_t *__restrict__ P1, uint32_t *__restrict__ cut,
             Part *__restrict__ part) {
    __shared__ uint32_t s_c[2 * kSplitThreads];
    __shared__ Cand s_v[2 * kSplitThreads];
    const int tid = threadIdx.x;
    const uint64_t tile_start = (uint64_t)blockIdx.x * kSplitTile;
    const uint64_t tile_end = min(tile_start + kSplitTile, A);
    const uint64_t a0 = tile_start + (uint64_t)tid * kSplitItems;
    const uint64_t a_end = min(a0 + kSplitItems, tile_end);

    uint32_t head_c = kNone, tail_c = kNone;
    Cand head_b = no_cand(), tail_b = no_cand();
    if (a0 < tile_end) {
        uint32_t c = (uint32_t)upper_bound(aoff, C, (uint32_t)a0) - 1;
        uint32_t lo = f_lo[c], hi = f_hi[c];
        uint64_t ao = aoff[c], ae = ao + (hi - lo);
        uint64_t p1lo = P1[lo], S = P1[hi] - p1lo;
        uint64_t seg_start = a0;
        Cand best = no_cand();
        auto flush = [&](uint64_t seg_end) {
            if (ao >= a0 && ae <= a_end) {
                cut[c] = best.k;                       // whole cluster inside this thread
            } else if (seg_start == a0) {
                head_c = c; head_b = best;
            } else {
                tail_c = c; tail_b = best;
            }
        };
        for (uint64_t a = a0; a < a_end; a++) {
            if (a >= ae) {
                flush(a);
                c++;
                lo = f_lo[c]; hi = f_hi[c];
                ao = aoff[c]; ae = ao + (hi - lo);
                p1lo = P1[lo]; S = P1[hi] - p1lo;
                seg_start = a;
                best = no_cand();
            }
            const uint32_t k = (uint32_t)(a - ao);
            if (k >= 1) {
                const uint64_t i = lo + k;
                const uint64_t pm = P1[i - 1], p0 = P1[i], pp = P1[i + 1];
                if (p0 - pm < pp - p0) {               // t[i-1] < t[i]: cut between distinct values
                    const Cand cd = make_cand(hi - lo, S, p0 - p1lo, k);
                    if (better(cd, best)) best = cd;
                }
            }
        }
        flush(a_end);
        if (head_c != kNone && tail_c == kNone) { tail_c = head_c; tail_b = head_b; }  // idempotent duplicate
    }
    // block-level segmented argmax (Hillis-Steele over 2 entries per thread;
    // runs of one cluster are contiguous, so "same id d entries back" = same run)
    s_c[2 * tid] = head_c;
    s_v[2 * tid] = head_b;
    s_c[2 * tid + 1] = tail_c;
    s_v[2 * tid + 1] = tail_b;
    __syncthreads();
    for (int d = 1; d < 2 * kSplitThreads; d <<= 1) {
        Cand nv[2];
        bool upd[2];
#pragma unroll
        for (int h = 0; h < 2; h++) {
            const int e = 2 * tid + h;
            const uint32_t ce = s_c[e];
            upd[h] = false;
            if (ce != kNone && e >= d && s_c[e - d] == ce) {
                const Cand o = s_v[e - d];
                nv[h] = s_v[e];
                if (better(o, nv[h])) { nv[h] = o; upd[h] = true; }
            }
        }
        __syncthreads();
#pragma unroll
        for (int h = 0; h < 2; h++)
            if (upd[h]) s_v[2 * tid + h] = nv[h];
        __syncthreads();
    }
#pragma unroll
    for (int h = 0; h < 2; h++) {
        const int e = 2 * tid + h;
        const uint32_t ce = s_c[e];
        if (ce == kNone) continue;
        if (e + 1 < 2 * kSplitThreads && s_c[e + 1] == ce) continue;   // not the run's last entry
        const uint64_t ao = aoff[ce], ae = ao + (f_hi[ce] - f_lo[ce]);
        if (ao >= tile_start && ae <= tile_end) {
            cut[ce] = s_v[e].k;
        } else {
            const int slot = (ao <= tile_start) ? 0 : 1;   // first cluster of the tile -> slot 0
            part[2 * (uint64_t)blockIdx.x + slot] = Part{s_v[e], ce};
        }
    }
}

__device__ __forceinline__ Cand shfl_cand(const Cand &a, int src) {
    Cand r;
    r.f = __shfl_sync(0xffffffffu, a.f, src);
    const uint64_t lo = __shfl_sync(0xffffffffu, (uint64_t)a.absD, src);
    const uint64_t hi = __shfl_sync(0xffffffffu, (uint64_t)(a.absD >> 64), src);
    r.absD = ((u128)hi << 64) | lo;
    r.p = __shfl_sync(0xffffffffu, a.p, src);
    r.k = __shfl_sync(0xffffffffu, a.k, src);
    return r;
}

__global__ void __launch_bounds__(256)
fixup_kernel(const uint32_t *__restrict__ f_lo, const uint32_t *__restrict__ f_hi, const uint32_t *__restrict__ aoff,
             uint32_t C, const Part *__restrict__ part, uint32_t *__restrict__ cut) {
    const uint64_t c = ((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int lane = threadIdx.x & 31;
    if (c >= C) return;
    const uint64_t ao = aoff[c], ae = ao + (f_hi[c] - f_lo[c]);
    const uint64_t j0 = ao / kSplitTile, j1 = (ae - 1) / kSplitTile;
    if (j0 == j1) return;
    Cand best = no_cand();
    for (uint64_t j = j0 + lane; j <= j1; j += 32) {
        const int slot = (j == j0 && ao != j0 * kSplitTile) ? 1 : 0;
        const Cand v = part[2 * j + slot].cand;
        if (better(v, best)) best = v;
    }
#pragma unroll
    for (int o = 16; o; o >>= 1) {
        const Cand v = shfl_cand(best, lane ^ o);
        if (better(v, best)) best = v;
    }
    if (lane == 0) cut[c] = best.k;
}

// ---------------------------------------------------------------- a4: decide
struct DecideArgs {
    const uint32_t *f_lo, *f_hi, *cut;
    uint32_t C;
    const uint64_t *P1;
    const u128 *P2;
    const uint32_t *t;
    uint8_t *flags;
    uint64_t *cnt_sz;
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

__global__ void __launch_bounds__(256) decide_kernel(DecideArgs a) {
    const uint64_t c = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (c >= a.C) return;
    const uint32_t lo = a.f_lo[c], hi = a.f_hi[c], k = a.cut[c];
    const uint32_t mid = lo + k;
    const uint64_t n = hi - lo, nL = k, nR = n - k;
    const uint64_t S = a.P1[hi] - a.P1[lo], SL = a.P1[mid] - a.P1[lo], SR = S - SL;
    const u128 Q = a.P2[hi] - a.P2[lo], QL = a.P2[mid] - a.P2[lo], QR = Q - QL;
    const u128 V = (u128)n * Q - (u128)S * S;
    const u128 VL = (u128)nL * QL - (u128)SL * SL, VR = (u128)nR * QR - (u128)SR * SR;
    // Eq. 7: tau_old = m * Xbar, m from Eq. 3
    const double mu = __ddiv_rn(rn64(S), rn64(n));
    const double tau_old = __dmul_rn(eq3_m(V, S, a.k2, a.clamp), mu);
    // Eq. 8 with Eq. 6 (corrected numerator) over {L, R}, c from the parent's total
    const double muL = __ddiv_rn(rn64(SL), rn64(nL)), muR = __ddiv_rn(rn64(SR), rn64(nR));
    const double dVL = rn128(VL), dVR = rn128(VR);
    const double w = __ddiv_rn(__dmul_rn(a.eps, rn64(S)), a.z);
    const double cc = __dmul_rn(w, w);
    const double ssum = __dadd_rn(__dsqrt_rn(__dmul_rn(muL, dVL)), __dsqrt_rn(__dmul_rn(muR, dVR)));
    const double g = __ddiv_rn(ssum, cc);
    const double mL = eq6_m(g, muL, dVL, a.clamp), mR = eq6_m(g, muR, dVR, a.clamp);
    const double tau_new = __dadd_rn(__dmul_rn(mL, muL), __dmul_rn(mR, muR));
    uint64_t cs = 0;
    if (k != 0 && tau_new < tau_old) {                  // strict
        a.flags[mid] = 1;
        const bool ntL = nontrivial(a.t, lo, mid), ntR = nontrivial(a.t, mid, hi);
        cs = ((uint64_t)(ntL + ntR) << 32) | (uint64_t)((ntL ? nL : 0) + (ntR ? nR : 0));
    }
    a.cnt_sz[c] = cs;
}

// ---------------------------------------------------------------- frontier bookkeeping
__global__ void group_flags_kernel(const uint32_t *goff, uint32_t K, uint8_t *flags) {
    const uint64_t g = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (g < K && goff[g] < goff[g + 1]) flags[goff[g]] = 1;
}

static int read_frontier_total(Ctx &c, uint64_t &C, uint64_t &A) {
    uint64_t tot = 0;
    CK(cudaMemcpyAsync(&tot, &c.scalars->frontier_total, sizeof(uint64_t), cudaMemcpyDeviceToHost, c.stream));
    CK(cudaStreamSynchronize(c.stream));
    C = tot >> 32;
    A = tot & 0xFFFFFFFFull;
    return STEM_OK;
}

int stem_only_leaves(Ctx &c, uint64_t n, uint32_t K) {
    CK(cudaMemsetAsync(c.flags, 0, n + 1, c.stream));
    group_flags_kernel<<<(unsigned)((K + 255) / 256), 256, 0, c.stream>>>(c.goff, K, c.flags);
    c.launches++;
    CK(cudaGetLastError());
    return STEM_OK;
}

int root_levels(Ctx &c, uint64_t n, uint32_t K, double eps, double z, double k2, int clamp) {
    cudaStream_t st = c.stream;
    CKS(stem_only_leaves(c, n, K));
    // initial frontier: non-trivial kernel groups, in kernel order
    {
        CKS(c.ensure(c.f_lo[0], c.cap_flo[0], sizeof(uint32_t) * ((uint64_t)K + 1)));
        CKS(c.ensure(c.f_hi[0], c.cap_fhi[0], sizeof(uint32_t) * ((uint64_t)K + 1)));
        CKS(c.ensure(c.f_aoff[0], c.cap_faoff[0], sizeof(uint32_t) * ((uint64_t)K + 1)));
        CKS(c.ensure(c.scan_scratch, c.cap_scan, (scan_tiles(K) + 1) * sizeof(uint64_t)));
        const uint32_t *goff = c.goff, *t = c.t_sorted;
        uint32_t *nlo = c.f_lo[0], *nhi = c.f_hi[0], *nao = c.f_aoff[0];
        exclusive_scan<uint64_t>(
            [goff, t] __device__(uint64_t g) -> uint64_t {
                const uint32_t lo = goff[g], hi = goff[g + 1];
                return nontrivial(t, lo, hi) ? ((1ull << 32) | (hi - lo)) : 0ull;
            },
            [nlo, nhi, nao, goff] __device__(uint64_t g, uint64_t pre, uint64_t v) {
                if (!v) return;
                const uint32_t idx = (uint32_t)(pre >> 32);
                nlo[idx] = goff[g];
                nhi[idx] = goff[g + 1];
                nao[idx] = (uint32_t)pre;
            },
            (uint64_t)K, (uint64_t *)c.scan_scratch, &c.scalars->frontier_total, st, &c.launches);
        CK(cudaGetLastError());
    }
    uint64_t C = 0, A = 0;
    CKS(read_frontier_total(c, C, A));
    int cur = 0;
    uint32_t levels = 0;
    while (C > 0) {
        levels++;
        c.stats.active_rows += A;
        const uint64_t ntiles = (A + kSplitTile - 1) / kSplitTile;
        CKS(c.ensure(c.cut, c.cap_cut, sizeof(uint32_t) * C));
        CKS(c.ensure(c.cnt_sz, c.cap_cntsz, sizeof(uint64_t) * C));
        CKS(c.ensure(c.split_part, c.cap_part, sizeof(Part) * 2 * ntiles));
        CKS(c.ensure(c.scan_scratch, c.cap_scan, (scan_tiles(C) + 1) * sizeof(uint64_t)));
        const int nxt = cur ^ 1;
        // children are at most 2 per cluster
        CKS(c.ensure(c.f_lo[nxt], c.cap_flo[nxt], sizeof(uint32_t) * 2 * C));
        CKS(c.ensure(c.f_hi[nxt], c.cap_fhi[nxt], sizeof(uint32_t) * 2 * C));
        CKS(c.ensure(c.f_aoff[nxt], c.cap_faoff[nxt], sizeof(uint32_t) * 2 * C));
        const int tk_s = c.stage_begin("root_split");
        split_kernel<<<(unsigned)ntiles, kSplitThreads, 0, st>>>(c.f_lo[cur], c.f_hi[cur], c.f_aoff[cur], (uint32_t)C, A,
                                                                c.P1, c.cut, (Part *)c.split_part);
        fixup_kernel<<<(unsigned)((C * 32 + 255) / 256), 256, 0, st>>>(c.f_lo[cur], c.f_hi[cur], c.f_aoff[cur],
                                                                       (uint32_t)C, (const Part *)c.split_part, c.cut);
        c.launches += 2;
        c.stage_end(tk_s, 8 * A + 4 * C * 3);
        const int tk_d = c.stage_begin("root_decide");
        DecideArgs da{c.f_lo[cur], c.f_hi[cur], c.cut, (uint32_t)C, c.P1, c.P2, c.t_sorted, c.flags, c.cnt_sz,
                      eps, z, k2, clamp};
        decide_kernel<<<(unsigned)((C + 255) / 256), 256, 0, st>>>(da);
        c.launches += 1;
        c.stage_end(tk_d, 96 * C);
        const int tk_c = c.stage_begin("root_compact");
        CK(cudaGetLastError());
        const uint32_t *flo = c.f_lo[cur], *fhi = c.f_hi[cur], *fcut = c.cut, *t = c.t_sorted;
        const uint64_t *cs = c.cnt_sz;
        uint32_t *nlo = c.f_lo[nxt], *nhi = c.f_hi[nxt], *nao = c.f_aoff[nxt];
        exclusive_scan<uint64_t>(
            [cs] __device__(uint64_t i) -> uint64_t { return cs[i]; },
            [flo, fhi, fcut, t, nlo, nhi, nao] __device__(uint64_t i, uint64_t pre, uint64_t v) {
                if (!v) return;
                uint32_t idx = (uint32_t)(pre >> 32), off = (uint32_t)pre;
                const uint32_t lo = flo[i], hi = fhi[i], mid = lo + fcut[i];
                if (nontrivial(t, lo, mid)) {
                    nlo[idx] = lo; nhi[idx] = mid; nao[idx] = off;
                    idx++; off += mid - lo;
                }
                if (nontrivial(t, mid, hi)) {
                    nlo[idx] = mid; nhi[idx] = hi; nao[idx] = off;
                }
            },
            C, (uint64_t *)c.scan_scratch, &c.scalars->frontier_total, st, &c.launches);
        c.stage_end(tk_c, 8 * C + 24 * C);
        CK(cudaGetLastError());
        CKS(read_frontier_total(c, C, A));
        cur = nxt;
    }
    c.stats.levels = levels;
    return STEM_OK;
}

}  // namespace sr
