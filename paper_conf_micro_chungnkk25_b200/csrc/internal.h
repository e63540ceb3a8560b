// internal.h -- host-side context and stage entry points of libstemroot.
#pragma once
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <vector>
#include <cuda_runtime.h>

#include "../../include/stemroot.h"
#include "common.cuh"
#include "scan.cuh"

#define CK(x)                                              \
    do {                                                   \
        cudaError_t e_ = (x);                              \
        if (e_ != cudaSuccess) {                           \
            sr::last_cuda_error() = e_;                    \
            return e_ == cudaErrorMemoryAllocation ? STEM_E_NOMEM : STEM_E_CUDA; \
        }                                                  \
    } while (0)

#define CKS(x)                                             \
    do {                                                   \
        int s_ = (x);                                      \
        if (s_ != STEM_OK) return s_;                      \
    } while (0)

namespace sr {

cudaError_t &last_cuda_error();

// Device-resident scalars of one plan call (one cudaMemcpy brings them home).
struct DevScalars {
    uint32_t max_t, err, tile_counter, pad0;
    uint64_t scan_total64;        // generic scan total
    uint64_t scan_total64b;       // second scan total (coarse key bases)
    uint64_t frontier_total;      // packed (count << 32 | rows) of the next frontier
    uint64_t ftot[2];             // ROOT levels: packed totals of the ping-pong frontiers
    uint64_t n_leaves;            // leaves after compaction
    uint64_t total_m;             // sum of m_i
    uint64_t sum_q;               // sum_i floor(n_i U_i / m_i)
    uint64_t T;                   // exact total time
    uint32_t limit_err, pad1;
    uint32_t big_count, pad2;     // big-cluster (cluster, segment) entries of the current level
    double ssum;                  // RN(exact sum sqrt(mu V)) (global scope)
    double g;                     // Ssum / c (global scope)
    double est_frac, var_sum;     // sum rn(r_i)/m_i, sum rn(V_i)/m_i
    alignas(16) uint64_t wide_total[4];   // total of a wide (struct) scan
    uint64_t red7[8];                     // multi-GPU reduction staging
    unsigned long long local_rows;        // rows scanned below the frontier (local subtrees)
    unsigned long long split_chunks, split_scanned;   // big-cluster chunks bounded / scanned row by row
    uint32_t local_depth, amb_count;      // deepest ROOT level of a local subtree; ambiguous samples
    uint32_t km_nsub[4];                  // split = 3: subproblems [short, long][current / next D&C round]
    uint32_t nc_queue[2];                 // nearest-centre descent: next cluster of the level's work queue (by level parity)
};

constexpr int kMaxCand = 64;     // packed sort: most candidate rows per sample (one u64 mask)

constexpr int kFixDigits = 6;     // 6 x 32-bit digits in u64 lanes, LSB 2^-72
constexpr int kFixLsb = 72;

// Optional per-stage CUDA-event timing (stem_ctx_enable_timing): each stage
// brackets its launches with two events on the plan's stream.
struct StageAgg {
    const char *name;
    double ms;
    uint64_t bytes;       // algorithmic bytes, summed over occurrences
    uint32_t launches, count;
};

struct Timing {
    bool on = false;
    struct Pending { const char *name; cudaEvent_t a, b; uint64_t bytes; uint32_t launches; };
    std::vector<cudaEvent_t> pool;
    size_t used = 0;
    std::vector<Pending> pend;
    std::vector<StageAgg> agg;
    cudaEvent_t get() {
        if (used == pool.size()) {
            cudaEvent_t e;
            cudaEventCreate(&e);
            pool.push_back(e);
        }
        return pool[used++];
    }
    void reset() { used = 0; pend.clear(); agg.clear(); }
    void finish() {   // stream already synchronised
        if (getenv("STEMROOT_GAPS")) {   // analysis: device idle before each stage (stderr)
            double tot = 0.0;
            for (size_t i = 1; i < pend.size(); i++) {
                float g = 0.f;
                cudaEventElapsedTime(&g, pend[i - 1].b, pend[i].a);
                if (g > 0.f) tot += g;
                if (g > 0.02f) fprintf(stderr, "gap %.3f ms before %s\n", g, pend[i].name);
            }
            float span = 0.f;
            if (!pend.empty()) cudaEventElapsedTime(&span, pend.front().a, pend.back().b);
            fprintf(stderr, "gaps total %.3f ms, stage span %.3f ms\n", tot, span);
        }
        for (auto &p : pend) {
            float ms = 0.f;
            cudaEventElapsedTime(&ms, p.a, p.b);
            StageAgg *g = nullptr;
            for (auto &x : agg) if (!strcmp(x.name, p.name)) g = &x;
            if (!g) { agg.push_back(StageAgg{p.name, 0.0, 0, 0, 0}); g = &agg.back(); }
            g->ms += ms; g->bytes += p.bytes; g->launches += p.launches; g->count++;
        }
        pend.clear();
    }
    ~Timing() { for (auto e : pool) cudaEventDestroy(e); }
};

class Comm;   // dist.cu: multi-GPU collectives (NCCL or in-process loopback)

struct Ctx {
    int device = 0;
    Comm *comm = nullptr;          // non-NULL inside stem_root_plan_dist
    uint32_t kid_base = 0;         // global id of local kernel 0 (dist: first owned kernel)
    int sms = 148;
    cudaStream_t stream = nullptr;
    cudaStream_t side = nullptr;                 // ROOT: the small-cluster split runs beside the big path
    cudaEvent_t ev_fork = nullptr, ev_join = nullptr;
    cudaStream_t vside = nullptr;                // ROOT: the value-histogram levels run beside the row levels
    cudaEvent_t ev_vfork = nullptr, ev_vjoin = nullptr;
    uint64_t *h_vr = nullptr;                    // pinned: value-level frontier totals (ring)
    uint64_t *h_vcount = nullptr;                // pinned: distinct values of the dense groups
    cudaEvent_t ev_vcount = nullptr;
    cudaEvent_t ev_vr[8] = {nullptr, nullptr, nullptr, nullptr, nullptr, nullptr, nullptr, nullptr};
    uint64_t *h_lvl = nullptr;                     // pinned: per-level frontier totals (ring of kLvlRing)
    cudaEvent_t ev_lvl[4] = {nullptr, nullptr, nullptr, nullptr};
    uint32_t launches = 0;
    stem_stats stats{};
    Timing timing;
    // stage bracket: returns an index to pass to stage_end (or -1 when timing is off)
    int stage_begin(const char *name) {
        if (!timing.on) return -1;
        cudaEvent_t a = timing.get(), b = timing.get();
        cudaEventRecord(a, stream);
        timing.pend.push_back(Timing::Pending{name, a, b, 0, launches});
        return (int)timing.pend.size() - 1;
    }
    void stage_end(int tok, uint64_t bytes) {
        if (tok < 0) return;
        auto &p = timing.pend[tok];
        cudaEventRecord(p.b, stream);
        p.bytes = bytes;
        p.launches = launches - p.launches;
    }

    // ---- workspace (grow-only)
    template <class T>
    int ensure(T *&p, size_t &cap, size_t bytes) {
        if (bytes <= cap) return STEM_OK;
        if (p) cudaFree(p);
        p = nullptr;
        cap = 0;
        size_t b = bytes + bytes / 8 + 256;
        cudaError_t e = cudaMalloc((void **)&p, b);
        if (e != cudaSuccess) { last_cuda_error() = e; p = nullptr; return STEM_E_NOMEM; }
        cap = b;
        return STEM_OK;
    }
    int ensure_all(uint64_t n, uint32_t K, uint32_t n_metrics);
    void release();

    // input copies when the trace is on the host
    uint32_t *in_kid = nullptr, *in_t = nullptr; size_t cap_in_kid = 0, cap_in_t = 0;
    double *in_met = nullptr; size_t cap_in_met = 0;
    // sort
    uint64_t *keys[2] = {nullptr, nullptr}; size_t cap_keys[2] = {0, 0};
    uint32_t *vals[2] = {nullptr, nullptr}; size_t cap_vals[2] = {0, 0};
    uint32_t *t_sorted = nullptr, *row_sorted = nullptr; size_t cap_ts = 0, cap_rs = 0;
    // packed sort (sort.cu): row_sorted holds the low pack_s bits of the row;
    // pack_h = candidate rows per sample (0: payload mode, row_sorted = rows)
    int pack_s = 0;
    uint32_t pack_h = 0;
    const uint32_t *sort_kid = nullptr, *sort_t = nullptr, *sort_row_in = nullptr;
    void *amb = nullptr; size_t cap_amb = 0;                   // ambiguous-sample entries
    uint32_t *kid_count = nullptr, *goff = nullptr; size_t cap_kc = 0, cap_goff = 0;
    uint32_t *kid_max = nullptr; size_t cap_kmax = 0;          // per-kernel max t
    uint64_t *key_base = nullptr; size_t cap_kbase = 0;        // [K + 1] offset-key bases
    uint64_t *key_base_c = nullptr; size_t cap_kbase_c = 0;    // [K + 1] coarse (2^24) bases
    uint32_t *key_base_s = nullptr; size_t cap_kbase_s = 0;    // [K + 1] chosen bases >> shift
    uint32_t *tailh = nullptr; size_t cap_tailh = 0;           // [K][256] rows per (kernel, t >> 24)
    uint32_t *kid_tab = nullptr; size_t cap_kid_tab = 0;       // key >> 16 -> kernel
    uint32_t *sort_mode = nullptr; size_t cap_sort_mode = 0;   // ranking mode per pass
    uint64_t *sort_gbase = nullptr; size_t cap_sort_gbase = 0; // [pass][256] digit bases
    uint64_t *hist = nullptr; size_t cap_hist = 0;
    void *sort_status = nullptr; size_t cap_status = 0;
    void *tile_hist = nullptr; size_t cap_tile_hist = 0;   // first pass: per-tile digit counts, group sums, offsets
    DevScalars *scalars = nullptr; size_t cap_scalars = 0;
    void *scan_scratch = nullptr; size_t cap_scan = 0;
    // sampled prefix moments (a2): PS1/PS2 every kChunk rows
    uint64_t *PS1 = nullptr; size_t cap_ps1 = 0;
    u128 *PS2 = nullptr; size_t cap_ps2 = 0;
    uint32_t *TB = nullptr; size_t cap_TB = 0;            // chunk-boundary pairs (t[32j-1], t[32j])
    void *chunk_sq = nullptr; size_t cap_chunk_sq = 0;
    // ROOT frontier (a3/a4)
    uint32_t *f_lo[2] = {nullptr, nullptr}, *f_hi[2] = {nullptr, nullptr}, *f_aoff[2] = {nullptr, nullptr};
    size_t cap_flo[2] = {0, 0}, cap_fhi[2] = {0, 0}, cap_faoff[2] = {0, 0};
    uint64_t *f_S[2] = {nullptr, nullptr}; size_t cap_fS[2] = {0, 0};
    u128 *f_Q[2] = {nullptr, nullptr}; size_t cap_fQ[2] = {0, 0};
    uint32_t *cut = nullptr; size_t cap_cut = 0;
    uint64_t *cut_SL = nullptr; size_t cap_cut_SL = 0;
    u128 *cut_QL = nullptr; size_t cap_cut_QL = 0;
    void *big_ent = nullptr, *big_part = nullptr, *big_thr = nullptr;
    size_t cap_big_ent = 0, cap_big_part = 0, cap_big_thr = 0;
    uint64_t *cnt_sz = nullptr; size_t cap_cntsz = 0;
    uint32_t *flags = nullptr; size_t cap_flags = 0;   // leaf-start bitmap: bit i & 31 of word i >> 5
    // leaves (a5/a6)
    uint32_t *leaf_lo = nullptr; size_t cap_leaf_lo = 0;
    uint64_t *leaf_m = nullptr, *leaf_moff = nullptr, *leaf_U = nullptr;
    size_t cap_leaf_m = 0, cap_leaf_moff = 0, cap_leaf_U = 0;
    uint8_t *leaf_census = nullptr; size_t cap_leaf_census = 0;
    uint32_t *leaf_kid = nullptr, *leaf_ord = nullptr; size_t cap_leaf_kid = 0, cap_leaf_ord = 0;
    uint64_t *fix_acc = nullptr; size_t cap_fix = 0;      // [K or 1][kFixDigits] lanes
    uint64_t *kern_T = nullptr; size_t cap_kern_T = 0;    // per-kernel T (scope 1)
    double *kern_g = nullptr; size_t cap_kern_g = 0;      // per-kernel g (scope 1)
    double *red_part = nullptr; size_t cap_red = 0;       // deterministic block partials
    // plan outputs (a7/a8)
    stem_cluster *out_clusters = nullptr; size_t cap_out_cl = 0;
    uint32_t *out_row = nullptr, *out_cluster = nullptr; size_t cap_out_row = 0, cap_out_cluster = 0;
    double *out_weight = nullptr; size_t cap_out_weight = 0;
    double host_est_metric[64];
    // multi-GPU (dist.cu)
    uint64_t *part_cnt = nullptr; size_t cap_part_cnt = 0;
    uint64_t *dist_cnt = nullptr; size_t cap_dist_cnt = 0;
    uint32_t *xfer_u32[3] = {nullptr, nullptr, nullptr}; size_t cap_xfer_u32[3] = {0, 0, 0};
    uint32_t *recv_u32[3] = {nullptr, nullptr, nullptr}; size_t cap_recv_u32[3] = {0, 0, 0};
    double *xfer_f64 = nullptr, *xfer_f64b = nullptr; size_t cap_xfer_f64 = 0, cap_xfer_f64b = 0;
    double *red_part2 = nullptr; size_t cap_red2 = 0;
    void *g_clusters = nullptr, *g_row = nullptr, *g_cluster = nullptr, *g_weight = nullptr;
    size_t cap_g_clusters = 0, cap_g_row = 0, cap_g_cluster = 0, cap_g_weight = 0;
    // split = 3 (kmeans.cu): distinct-value starts, DP tables, groups per cluster
    uint32_t *km_dpos = nullptr, *km_arg = nullptr, *km_ngrp = nullptr;
    size_t cap_km_dpos = 0, cap_km_arg = 0, cap_km_ngrp = 0;
    uint64_t *km_dP = nullptr; size_t cap_km_dP = 0;
    double *km_F = nullptr; size_t cap_km_F = 0;
    void *km_meta = nullptr, *km_sub = nullptr; size_t cap_km_meta = 0, cap_km_sub = 0;
    void *peer_dst = nullptr; size_t cap_peer_dst = 0;
    // multi-GPU kernels larger than a rank's share (root.cu root_values, dist.cu)
    void *vr_P = nullptr, *vr_work = nullptr; size_t cap_vr_P = 0, cap_vr_work = 0;
    void *gi_buf = nullptr; size_t cap_gi_buf = 0;
    void *dn_sel = nullptr, *dn_meta = nullptr, *dn_val = nullptr;   // value path of repeated-time groups
    size_t cap_dn_sel = 0, cap_dn_meta = 0, cap_dn_val = 0;
    void *gi_tab = nullptr, *gi_rec = nullptr, *gi_all = nullptr, *gi_val = nullptr;   // histograms, tables
    size_t cap_gi_tab = 0, cap_gi_rec = 0, cap_gi_all = 0, cap_gi_val = 0;
    const uint8_t *fixed_kernel = nullptr;                  // local kernels whose leaves are given (no ROOT)
    const uint32_t *fixed_cuts = nullptr; uint64_t n_fixed_cuts = 0;   // their inner leaf starts: (local kernel, row in group)
    const uint32_t *ord_off = nullptr;                      // per local kernel: ordinal of its first local leaf   // fused exchange: the owners' windows (PeerDst)
    uint64_t row_bases[65] = {0};
    uint64_t n_local_rows = 0;
    // metric_bounds (metric.cu): leaf table (first leaf per kernel, lo_ns, n, m), per-leaf sums
    uint32_t *mb_first = nullptr, *mb_lo = nullptr, *mb_gkid = nullptr, *mb_leaf_of = nullptr;
    size_t cap_mb_first = 0, cap_mb_lo = 0, cap_mb_gkid = 0, cap_mb_leaf_of = 0;
    uint64_t *mb_n = nullptr, *mb_gm = nullptr; size_t cap_mb_n = 0, cap_mb_gm = 0;
    const uint64_t *mb_m = nullptr;                  // leaf_m (single GPU) or mb_gm (gathered)
    double *mb_acc = nullptr, *mb_part = nullptr; size_t cap_mb_acc = 0, cap_mb_part = 0;
    void *mb_rec = nullptr; size_t cap_mb_rec = 0;
    bool have_mbounds = false;
    double host_true_metric[64], host_bound_metric[64];

    // host plan: with want_host the single-GPU path allocates the caller's plan
    // block as soon as its size is known and copies the cluster records into it
    // on dstream while the samples are drawn (capi.cu plan_block_begin / to_host)
    bool want_host = false;
    void *early_plan = nullptr;                 // PlanBlock (capi.cu), or NULL
    cudaStream_t dstream = nullptr;
    cudaEvent_t ev_pack = nullptr, ev_d2h = nullptr;
    cudaEvent_t ev_h2d[8] = {nullptr, nullptr, nullptr, nullptr, nullptr, nullptr, nullptr, nullptr};
    cudaEvent_t ev_pre = nullptr;
    bool early_packed = false;

    // last plan
    bool have_plan = false;
    uint64_t n = 0, n_leaves = 0, n_samples = 0, T = 0;
    uint64_t n_samples_global = 0;
    uint32_t K = 0, n_metrics = 0;
    double est_total = 0, bound = 0, eps = 0, z = 0;
};

// host wait for c.stream: with a communicator, polls for peer failures and the
// comm timeout (STEM_E_NCCL) instead of blocking forever (dist.cu)
int sync_stream(Ctx &c);
// multi-GPU: agree on a local status across ranks (identity without a communicator)
int dist_checkpoint(Ctx &c, int status);
// multi-GPU collectives on c.comm (dist.cu); device buffers, in place, sums
int comm_rank(const Comm *c);
int comm_world(const Comm *c);
int comm_allgather_host(Ctx &c, const uint64_t *mine, size_t count, uint64_t *all);
int comm_alltoallv(Ctx &c, const void *send, const uint64_t *scnt, const uint64_t *sdsp, void *recv,
                   const uint64_t *rcnt, const uint64_t *rdsp, size_t elem);
int dist_allreduce_u64(Ctx &c, uint64_t *buf, size_t count);
int dist_allreduce_f64(Ctx &c, double *buf, size_t count);
int dist_metric_sums(Ctx &c, const double *metrics_local, uint32_t nm, uint64_t S, double *out);

// stages
// h_kid/h_t (optional): the trace is in host memory and kid/t are its device
// copies to fill; the copies go in chunks and the pre-pass consumes each chunk
// as it lands (host-to-device traffic overlapped with the pre-pass)
int sort_trace(Ctx &c, const uint32_t *kid, const uint32_t *t, const uint32_t *row_in, uint64_t n,
               uint32_t K, bool allow_pack, const uint32_t *h_kid = nullptr, const uint32_t *h_t = nullptr);                                                   // a1
int prefix_moments(Ctx &c, uint64_t n);                                                        // a2
int root_levels(Ctx &c, uint64_t n, uint32_t K, double eps, double z, double k2, int clamp,
                int split, uint64_t seed);   // a3, a4 (split: 0 exact 2-means, 1 Lloyd, 2 k-means++ Lloyd)
int stem_only_leaves(Ctx &c, uint64_t n, uint32_t K);
// ROOT over a histogram of distinct values per group (root.cu): vflag[u] = 1 where a leaf starts
int root_values(Ctx &c, const uint32_t *vt, const uint64_t *vcnt, const uint32_t *goffv, uint32_t G, uint64_t D,
                double eps, double z, double k2, int clamp, uint8_t *vflag);
// One pipelined run of the value-histogram ROOT (root.cu): setup enqueues the
// first frontier on stream s, pump advances the levels (block = false: never
// waits), finish completes them.
struct VrSource {
    const uint32_t *kc = nullptr;      // [D] rows before value u
    const uint64_t *Ps = nullptr;      // [D] sum of t before value u
    const u128 *Pq = nullptr;          // [D] sum of t^2 before value u (histogram input; nullptr: from the rows)
    const uint32_t *goffv = nullptr;   // [G + 1] first value of each group
    const uint32_t *dgrp = nullptr;    // dense path: group j's kernel group (rows from goff, PS1/PS2)
    const uint32_t *goff = nullptr;
    uint32_t G = 0;
};
struct VrRun {
    Ctx &c;
    cudaStream_t st = nullptr;
    uint64_t D = 0;
    uint64_t enq = 0, done = 0;
    bool finished = false;
    uint32_t launches = 0, levels = 0;
    struct VrDevStore { alignas(16) unsigned char b[256]; } devs;
    int setup(const VrSource &src, uint64_t D, double eps, double z, double k2, int clamp, uint8_t *vflag,
              cudaStream_t s);
    int enqueue_one();
    int pump(bool block);
    int finish(uint64_t *active_rows);
};
// Kernel groups with many repeated times take the value path (root.cu)
struct DensePath {
    Ctx &c;
    VrRun run{c};
    bool on = false;
    int phase = 0;                   // 1: distinct count queued, 2: levels running
    const uint8_t *sel_ = nullptr;   // per group: 0 row path, 1 fixed leaves, 2 value path
    uint32_t *dgrp = nullptr, *dsegf = nullptr, *goffv = nullptr, *segcnt = nullptr, *segoff = nullptr;
    uint32_t *vpos = nullptr;
    uint8_t *vflag = nullptr;
    uint64_t D_ = 0;
    uint32_t Gd = 0, NS = 0;         // dense groups, their windows (kWinRows rows, one warp each)
    uint64_t n_ = 0;
    unsigned grid = 0;
    bool sync_mode = false;
    cudaStream_t vs_ = nullptr;
    uint64_t act_ = 0;
    double eps_ = 0, z_ = 0, k2_ = 0;
    int clamp_ = 0;
    int start(uint64_t n, uint32_t K, double eps, double z, double k2, int clamp);
    int build();
    int pump();
    int finish(uint32_t *flags);
};
// split = 3: ROOT with exact optimal 1-D k-means splits into kk groups (kmeans.cu, R29)
int root_levels_kmeans(Ctx &c, uint64_t n, uint32_t K, double eps, double z, double k2, int clamp, uint32_t kk);
int histogram_kernels(Ctx &c, const uint32_t *kid, const uint32_t *t, uint64_t n, uint32_t K,
                      uint32_t *tailh, bool zero = true, cudaStream_t pst = nullptr, uint16_t *tileh = nullptr,
                      uint64_t tile0 = 0);   // pre-pass only (tileh: the first sort pass's tile histograms too)   // pre-pass only
int run_plan_dist(Ctx &c, Comm &comm, const stem_trace *tr, uint64_t row_base, double eps, double conf,
                  const stem_opts &o, int local_status);
// capi.cu: allocate the host plan block for L clusters, S samples (c.early_plan);
// returns the device-to-host destination of the cluster records
int plan_block_begin(Ctx &c, uint64_t L, uint64_t S, uint32_t nm, stem_cluster **clusters_dst, uint32_t **row_dst,
                     uint32_t **cl_dst, double **w_dst);
void plan_block_abort(Ctx &c);
int leaves_and_plan(Ctx &c, uint64_t n, uint32_t K, const double *metrics, uint32_t n_metrics, double eps,
                    double z, double k2, const stem_opts &o, const uint32_t *tr_kid = nullptr,
                    const uint32_t *tr_t = nullptr, uint64_t tr_n = 0);                        // a5..a8
// a8 option metric_bounds (metric.cu): true totals and bounds into host_true/bound_metric
int metric_bounds_local(Ctx &c, uint64_t L, uint32_t K, uint64_t n_sorted, const uint32_t *kid, const uint32_t *t,
                        const double *met, uint64_t n_trace, uint32_t nm, double z);
int metric_bounds_dist(Ctx &c, uint64_t L_local, uint64_t n_sorted, uint32_t K_global, const uint32_t *kid,
                       const uint32_t *t, const double *met, uint64_t n_home, uint32_t nm, double z);

}  // namespace sr
