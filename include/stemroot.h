/*
 * stemroot.h -- C ABI of the B200-native STEM+ROOT sampling-plan builder.
 *
 * The library turns a kernel-invocation trace (kernel id, integer execution
 * time in ns, optional metric columns) into a sampling plan, following the
 * problem statement of Chung et al., "Swift and Trustworthy Large-Scale GPU
 * Simulation with Fine-Grained Error Modeling and Hierarchical Clustering",
 * MICRO'25 (cited as P:L<n> = line n of the paper text, PAPER.md):
 *   step a1  group invocations by kernel name ............ P:L101 (§3)
 *   step a2  prefix moments of t and t^2 ................. needed by Eq. 7/8
 *   step a3  ROOT split choice: k-means, k = 2 ........... P:L192, P:L258 (§3.4)
 *   step a4  ROOT accept iff tau_old > tau_new ........... Eq. 7/8
 *   step a5  leaf table (clusters) ....................... Fig. 6
 *   step a6  STEM sample sizes, joint KKT ................ Eq. 6, P:L169 (numerator
 *            corrected from the derivation), Eq. 5, Eq. 3
 *   step a7  random sampling with replacement ............ P:L120
 *   step a8  weighted-sum extrapolation + bound .......... P:L107, Eq. 4/5
 * Every step runs in hand-written sm_100a CUDA kernels; there is no CPU path.
 * The exact arithmetic order of every step is DESIGN.md §3 ("Readings").
 *
 * Conventions for every function:
 *  - Return value: STEM_OK (0) or a negative stem_status; no exception or
 *    abort crosses the ABI.  On error every output pointer is set to NULL.
 *  - Ownership: inputs are borrowed (read-only, caller-owned, valid for the
 *    call).  Plans returned in *out are allocated by the library in host
 *    memory and released only by stem_plan_free.  Device scratch belongs to a
 *    stem_ctx and lives until stem_ctx_destroy.
 *  - Synchrony: every call returns after the result is complete (the stream
 *    given in stem_opts.stream is synchronised before returning).
 *  - Threads: distinct stem_ctx objects may be used concurrently from
 *    distinct host threads; one stem_ctx must not be used concurrently.
 *  - Reproducibility: the plan is a pure function of (trace bytes, eps, z,
 *    seed, opts): integer outputs and sample rows are bit-identical to the
 *    test oracle; fp64 outputs agree with it to 1e-9 relative (all of them
 *    bit-identical run to run except true_metric / bound_metric).
 */
#ifndef STEMROOT_H
#define STEMROOT_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define STEMROOT_ABI_VERSION 5   /* 2: stem_opts.split; 3: split = 2 (k-means++ seeds);
                                    4: metric_bounds, true_metric, bound_metric; split = 3 and
                                    kmeans_k; stem_stats.owned_rows/world/fused_exchange;
                                    5: stem_stats.value_groups/value_count/value_levels */

#if defined(__GNUC__)
#define STEM_API __attribute__((visibility("default")))
#else
#define STEM_API
#endif

typedef enum stem_status {
    STEM_OK = 0,
    STEM_E_INVAL = -1,  /* NULL trace/out, eps or conf outside (0,1), n = 0, bad z/scope/metrics */
    STEM_E_RANGE = -2,  /* n >= 2^32, n_kernels = 0 or > 2^24, or some kernel_id >= n_kernels    */
    STEM_E_NOMEM = -3,  /* host or device allocation failed                                       */
    STEM_E_CUDA = -4,   /* a CUDA runtime call or kernel failed (no device, bad pointer, ...)     */
    STEM_E_NCCL = -5,   /* reserved for the multi-GPU entry point                                 */
    STEM_E_LIMIT = -6,  /* total sample count would reach 2^32, or some m_i >= 2^32; split = 3:
                           more than 256 exactly tied candidates in one k-means DP cell          */
    STEM_E_STATE = -7   /* stem_ctx_device_plan called before any successful plan on that ctx     */
} stem_status;

/* The trace.  Rows are kernel invocations in trace order; row index r is the
 * identity reported back in stem_plan.sample_row. */
typedef struct stem_trace {
    uint64_t        n;          /* rows, 1 <= n < 2^32                                         */
    uint32_t        n_kernels;  /* kernel ids are dense: 0 <= kernel_id[r] < n_kernels <= 2^24 */
    const uint32_t *kernel_id;  /* [n]  grouping key (one id per kernel name)           */
    const uint32_t *exec_ns;    /* [n]  execution time, integer ns (NSYS durations)     */
    uint32_t        n_metrics;  /* 0..64 metric columns extrapolated like time         */
    const double   *metrics;    /* [n_metrics][n] column-major, or NULL when n_metrics = 0      */
    int             device;     /* -1: all pointers are host memory (copied in by the library);
                                   >= 0: all pointers are device memory on this CUDA device     */
} stem_trace;

typedef struct stem_opts {
    uint64_t seed;           /* Philox4x32-10 key for the sample draws (R14)          */
    double   z;              /* 0: z = Phi^-1(1 - (1-conf)/2); > 0: use this z (1.96 = P:L126)  */
    int      scope;          /* sample-size solve over: 0 all leaves jointly (default),
                                1 each kernel's leaves, 2 each leaf alone by Eq. 3     */
    int      root;           /* 1: ROOT hierarchical clustering (default); 0: STEM only, one
                                cluster per kernel                                               */
    int      clamp_in_split; /* 1 (default): m >= 1 inside Eq. 7/8; 0: literal ceilings (R7)     */
    int      census_cap;     /* 1: a leaf whose m_i >= n_i takes all its n_i rows once (exact)   */
    int      split;          /* ROOT's sub-clustering ("a clustering method (e.g.,
                                k-means)", P:L258 k = 2): 0 (default) the exact optimal 2-means
                                cut (R5); 1 Lloyd's k-means, k = 2, from the (min, max)
                                centroids to its fixed point (R26); 2 the same Lloyd iteration
                                from k-means++ seeds (uniform c1, D^2-weighted c2) drawn with
                                Philox4x32-10 keyed by seed on (min t, max t, n) (R27), so the
                                tree depends on seed; 3 the exact optimal 1-D k-means with
                                kmeans_k groups per split (R29); other values: STEM_E_INVAL     */
    int      metric_bounds;  /* 1: also the exact total and the predicted relative error of each
                                metric column (Eq. 5 with the metric in place of t, P:L150-159,
                                P:L371; R28): stem_plan.true_metric / bound_metric.
                                0 (default): point estimates only, those two pointers are NULL  */
    int      kmeans_k;       /* split = 3: ROOT divides each cluster into min(kmeans_k, #distinct
                                values) groups by the exact optimal 1-D k-means ("any
                                number above 2 works well"; R29) and keeps them iff
                                Eq. 8 over the groups beats Eq. 7; 2..8 (default 3), ignored for
                                the other split rules                                            */
    void    *stream;         /* cudaStream_t to run on; NULL = the legacy default stream         */
} stem_opts;

/* One leaf of the ROOT tree: all rows of kernel_id with lo_ns <= t <= hi_ns. */
typedef struct stem_cluster {
    uint32_t kernel_id;
    uint32_t ordinal;        /* rank of the leaf within its kernel, by lo_ns                     */
    uint32_t lo_ns, hi_ns;   /* min and max execution time in the leaf                           */
    uint64_t n;              /* N_i, rows in the leaf                                            */
    uint64_t sum_ns;         /* exact sum of t over the leaf                                     */
    double   mean_ns;        /* mu_i = sum_ns / n                                                */
    double   std_ns;         /* population sigma_i (R3)                                */
    uint64_t m;              /* STEM sample size m_i >= 1                                        */
    uint32_t census;         /* 1: the samples are rows lo..hi of the leaf, each once            */
    uint32_t reserved;
} stem_cluster;

typedef struct stem_plan {
    uint64_t      n_clusters;
    stem_cluster *clusters;       /* [n_clusters], sorted by (kernel_id, ordinal)                 */
    uint64_t      n_samples;      /* sum of m_i                                                   */
    uint32_t     *sample_row;     /* [n_samples] trace row of each sample, ordered (cluster, j)   */
    uint32_t     *sample_cluster; /* [n_samples] index into clusters[]                            */
    double       *sample_weight;  /* [n_samples] n_i / m_i: invocations the sample stands for     */
    double        est_total_ns;   /* sum_i n_i * mean(sampled t)                 */
    uint64_t      true_total_ns;  /* exact T = sum of all t                                       */
    double        bound;          /* predicted error z*sqrt(sum_i V_i/m_i)/T <= eps (Eq. 5)       */
    double        eps, z;
    uint32_t      n_metrics;
    double       *est_metric;     /* [n_metrics] weighted-sum estimate of each metric total       */
    double       *true_metric;    /* [n_metrics] exact column sum (metric_bounds = 1), else NULL  */
    double       *bound_metric;   /* [n_metrics] z sqrt(sum_i V_ic/m_i)/|true_c| with V_ic =
                                     n_i^2 sigma_ic^2 of the metric over leaf i (R28); 0 for a
                                     zero-variance column, +inf when true_c = 0 and the variance
                                     is not (metric_bounds = 1), else NULL.  These two come from
                                     fp64 atomics: within 1e-12 relative run to run, not bitwise */
} stem_plan;

/* Device-resident view of the last plan built on a ctx (pointers owned by the
 * ctx, valid until the next plan call on it or stem_ctx_destroy). */
typedef struct stem_device_plan {
    uint64_t            n_clusters, n_samples;
    const stem_cluster *clusters;       /* device [n_clusters]                                  */
    const uint32_t     *sample_row;     /* device [n_samples]                                   */
    const uint32_t     *sample_cluster; /* device [n_samples]                                   */
    const double       *sample_weight;  /* device [n_samples]                                   */
    double              est_total_ns, bound, eps, z;
    uint64_t            true_total_ns;
    uint32_t            n_metrics;
    const double       *est_metric;     /* host [n_metrics]                                     */
    const double       *true_metric;    /* host [n_metrics], NULL unless metric_bounds          */
    const double       *bound_metric;   /* host [n_metrics], NULL unless metric_bounds          */
} stem_device_plan;

/* Counters of the last plan built on a ctx (for benchmarks and tests). */
typedef struct stem_stats {
    uint32_t key_bits;         /* bits of the (kernel, time) sort key                           */
    uint32_t sort_passes;      /* radix passes run                                             */
    uint32_t levels;           /* ROOT levels run (frontier iterations)                          */
    uint32_t kernel_launches;  /* CUDA kernels launched by the last plan call                    */
    uint64_t active_rows;      /* sum over levels of rows in the ROOT frontier                   */
    uint64_t n_clusters, n_samples;
    double   ssum;             /* RN(exact sum_i sqrt(mu_i V_i)) of the global KKT solve          */
    uint32_t pack_bits;        /* low row bits carried inside the sort key (0: row payload mode)  */
    uint32_t ambiguous_samples;/* samples whose row needed the run scan (packed mode)            */
    uint32_t coarse_bases;     /* 1: kernel key bases aligned to 2^24 (pass histograms from the pre-pass) */
    uint32_t reserved0;
    uint64_t split_chunks;     /* 32-row chunks of big clusters bounded, summed over ROOT levels   */
    uint64_t split_scanned;    /* of those, chunks scanned row by row (the rest pruned exactly)   */
    uint64_t owned_rows;       /* rows this ctx grouped and clustered: n on one GPU; in
                                  stem_root_plan_dist the rows of the kernels this rank owns
                                  after the exchange (max/mean over ranks = the imbalance)     */
    uint32_t world;            /* ranks of the communicator of the last plan (1 on one GPU)    */
    uint32_t fused_exchange;   /* 1: the last stem_root_plan_dist stored every row straight into
                                  its owner's receive window (peer memory over NVLink, CUDA IPC);
                                  0: grouped send/recv (STEMROOT_DIST_P2P=0, or no peer access) */
    uint32_t value_levels;     /* ROOT levels of the value-histogram path (0: not used)         */
    uint64_t value_groups;     /* kernel groups whose ROOT tree was built over their distinct
                                  values instead of their rows (split = 0: groups of
                                  >= STEMROOT_VALUE_ROWS rows whose times repeat; the tree is
                                  the same)                                    */
    uint64_t value_count;      /* distinct values of those groups                               */
} stem_stats;

/* Per-stage device time of the last plan (stem_ctx_enable_timing).  bytes is
 * the stage's algorithmic HBM traffic as DESIGN.md §6 defines it. */
typedef struct stem_stage_time {
    char     name[24];         /* e.g. "sort_pass_mid", "root_split"                            */
    double   ms;               /* summed CUDA-event time over the stage's occurrences            */
    uint64_t bytes;            /* summed algorithmic bytes                                       */
    uint32_t launches;         /* kernels launched by the stage                                  */
    uint32_t count;            /* occurrences (passes, levels)                                    */
} stem_stage_time;

typedef struct stem_ctx stem_ctx;

/* Fill *o with the defaults: seed 0, z 0, scope 0, root 1, clamp_in_split 1,
 * census_cap 0, split 0, metric_bounds 0, kmeans_k 3, stream NULL. */
STEM_API int stem_default_opts(stem_opts *o);

/* A workspace bound to one CUDA device; keeps device scratch between calls. */
STEM_API int  stem_ctx_create(int device, stem_ctx **out);
STEM_API void stem_ctx_destroy(stem_ctx *ctx);  /* NULL-safe */

/* Build the plan on ctx.  opts = NULL means defaults.  out = NULL keeps the
 * plan on the device only (read it with stem_ctx_device_plan); otherwise a
 * host copy is returned in *out.  conf is the two-sided confidence 1-alpha
 * (P:L124); it is ignored when opts->z > 0. */
STEM_API int stem_root_plan_ctx(stem_ctx *ctx, const stem_trace *trace, double eps, double conf,
                       const stem_opts *opts, stem_plan **out);

/* One-shot form of the paper's problem statement (north_star
 * stem_root_plan(trace, n, eps, conf)): a temporary ctx on trace->device
 * (device 0 for host traces), host plan in *out. */
STEM_API int stem_root_plan(const stem_trace *trace, double eps, double conf, const stem_opts *opts,
                   stem_plan **out);

STEM_API int stem_ctx_device_plan(const stem_ctx *ctx, stem_device_plan *view);
STEM_API int stem_ctx_stats(const stem_ctx *ctx, stem_stats *stats);

/* Bracket every stage of later plans on ctx with CUDA events (on = 1) or stop
 * (on = 0).  stem_ctx_stage_times copies up to cap records of the last plan
 * into out and the number available into *count. */
STEM_API int stem_ctx_enable_timing(stem_ctx *ctx, int on);
STEM_API int stem_ctx_stage_times(const stem_ctx *ctx, stem_stage_time *out, uint32_t cap, uint32_t *count);

STEM_API void        stem_plan_free(stem_plan *p);  /* frees everything in the plan; NULL-safe */
STEM_API const char *stem_strerror(int status);     /* static string, never NULL               */

/* ---- multi-GPU (one process or thread per GPU) ---------------------------
 * The trace is sharded by contiguous row ranges: rank r holds rows
 * [global_row_base_r, global_row_base_r + local_shard->n) (shards in rank
 * order, no gaps; a shard may be empty).  stem_root_plan_dist exchanges rows so
 * that every rank owns whole kernel groups (contiguous kernel-id ranges of
 * ~N/world rows, stem_owner_ranges) -- by default each row is stored straight
 * into its owner's receive window (CUDA-IPC peer memory over NVLink/NVSwitch;
 * STEMROOT_DIST_P2P=0, or peers without access, use grouped ncclSend/Recv) --
 * runs steps a1-a5 locally, reduces T and the exact KKT sum as integers
 * across ranks, samples locally, and gathers the plan on rank 0 (*out is set
 * on rank 0 only; other ranks get NULL and keep their own part, which
 * stem_ctx_device_plan then describes).  The plan is identical to
 * stem_root_plan on the unsharded trace for every world size (integers
 * bit-exact, fp64 sums within 1e-9 relative).  All ranks must call it
 * collectively with the same eps, conf, opts and n_kernels.
 * Failure semantics: rank-local errors (a bad shard, an allocation, a CUDA
 * error) are agreed across ranks before the next collective, so every rank
 * returns the same status; a peer that fails or disappears makes the others
 * return STEM_E_NCCL after STEMROOT_COMM_TIMEOUT_S seconds (default 600: the
 * NCCL communicator polls ncclCommGetAsyncError and aborts itself), after which
 * the communicator is unusable.
 * Entry point shape (a recorded choice): the communicator and
 * the workspace are objects created once and reused across plans; the
 * one-shot form (unique id, rank, world per call) is stem_comm_init_nccl +
 * stem_ctx_create + stem_root_plan_dist + the destroys. */
typedef struct stem_comm stem_comm;

/* 128 opaque bytes created by one rank and shared with all (e.g. broadcast
 * through torch.distributed); STEM_E_NCCL if libnccl.so.2 cannot be loaded. */
STEM_API int  stem_comm_nccl_unique_id(void *id_out);
/* NCCL communicator over NVLink/NVSwitch for (rank, world) on CUDA device. */
STEM_API int  stem_comm_init_nccl(const void *id, int rank, int world, int device, stem_comm **out);
/* world communicators sharing one device, to be driven by world host threads
 * (in-process test and emulation of the multi-rank logic on one GPU). */
STEM_API int  stem_comm_init_loopback(int world, int device, stem_comm **comms);
STEM_API void stem_comm_destroy(stem_comm *comm);   /* NULL-safe */
/* bounds[r] = first kernel id owned by rank r (bounds[world] = n_kernels):
 * the smallest k with (sum_{j<k} counts[j]) * world >= r * sum(counts).  Host only. */
STEM_API int  stem_owner_ranges(const uint64_t *counts, uint32_t n_kernels, int world, uint32_t *bounds);
STEM_API int  stem_root_plan_dist(stem_ctx *ctx, stem_comm *comm, const stem_trace *local_shard,
                                  uint64_t global_row_base, double eps, double conf, const stem_opts *opts,
                                  stem_plan **out);

/* z = Phi^-1(1 - (1-conf)/2), conf in (0,1); host computation. */
STEM_API int stem_z_from_conf(double conf, double *z_out);

#ifdef __cplusplus
}
#endif
#endif /* STEMROOT_H */
