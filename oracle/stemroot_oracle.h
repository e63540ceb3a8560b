/*
 * stemroot_oracle.h -- TEST INFRASTRUCTURE ONLY.
 *
 * The oracle is a plain, slow, single-threaded CPU implementation of the
 * STEM+ROOT sampling-plan hot path, written from PAPER.md (Chung et al.,
 * MICRO'25) and the readings listed in DESIGN.md.  Only tests/,
 * __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference
 * legs may load it.  It shares no code, header, table or constant with the
 * CUDA library under paper_conf_micro_chungnkk25_b200/ and include/.
 *
 * Citations: P:L<n> = /root/reference/PAPER.md line n.
 */
#ifndef STEMROOT_ORACLE_H
#define STEMROOT_ORACLE_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

enum { OR_OK = 0, OR_E_INVAL = -1, OR_E_RANGE = -2, OR_E_NOMEM = -3, OR_E_LIMIT = -6 };

typedef struct {
    uint64_t seed;           /* Philox key                                         */
    double   z;              /* z score; must be > 0 (the oracle never derives it) */
    int      scope;          /* 0 global joint KKT, 1 per kernel, 2 per leaf Eq.3  */
    int      root;           /* 1 ROOT on, 0 STEM only                             */
    int      clamp_in_split; /* 1: m >= 1 inside Eq.7/8; 0: literal ceilings       */
    int      census_cap;     /* 1: m_i >= n_i => take all n_i rows                 */
    int      split;          /* 0: exact optimal 2-means cut (R5); 1: Lloyd's k-means,
                                k = 2, from the (min, max) centroids (R26); 2: the
                                same from k-means++ seeds drawn with seed (R27); 3:
                                exact optimal 1-D k-means, k = kmeans_k (R29)       */
    int      metric_bounds;  /* 1: also true_metric and bound_metric (reading R28)   */
    int      kmeans_k;       /* split = 3: groups per ROOT split, 2..8               */
} or_opts;

/* Structure-of-arrays plan.  Everything is malloc'ed; free with or_plan_free. */
typedef struct {
    uint64_t  n_clusters;
    uint32_t *kernel_id, *ordinal, *lo_ns, *hi_ns;
    uint64_t *n, *sum_ns, *m;
    double   *mean_ns, *std_ns;
    uint8_t  *census;
    uint64_t  n_samples;
    uint32_t *sample_row, *sample_cluster;
    double   *sample_weight;
    double    est_total_ns;
    uint64_t  true_total_ns;
    double    bound, eps, z;
    uint32_t  n_metrics;
    double   *est_metric;        /* [n_metrics]                              */
    double    ssum;              /* RN(exact sum sqrt(mu_i V_i)), global     */
    uint32_t  max_depth;         /* deepest ROOT level reached (root = 0)    */
    double   *true_metric;       /* [n_metrics] exact column sums (metric_bounds), else NULL */
    double   *bound_metric;      /* [n_metrics] predicted relative error (R28), else NULL   */
} or_plan;

/* Whole plan (§3, Fig. 5).  kernel_id/exec_ns: [n];
 * metrics: column-major [n_metrics][n] or NULL.  Returns OR_* status. */
int  or_plan_build(uint64_t n, uint32_t n_kernels, const uint32_t *kernel_id,
                   const uint32_t *exec_ns, uint32_t n_metrics, const double *metrics,
                   double eps, const or_opts *opts, or_plan **out);
void or_plan_free(or_plan *p);

/* ---- pieces exposed for the pins in tests/test_oracle_pins.py ---- */
/* Philox4x32-10 (Salmon et al. SC'11 / Random123): out = Philox(ctr, key). */
void or_philox4x32_10(const uint32_t ctr[4], const uint32_t key[2], uint32_t out[4]);
/* Optimal 2-means cut of sorted t[0..n): returns k* in [1,n-1]
 * or 0 when no cut exists (n < 2 or all equal). */
uint64_t or_best_cut(const uint32_t *t_sorted, uint64_t n);
/* Lloyd's k-means with k = 2 on sorted t[0..n) ("k-means", P:L258 k = 2;
 * reading R26): returns the converged cut k in [1, n-1], 0 when no cut exists;
 * *iters gets the number of assignment steps. */
uint64_t or_lloyd_cut(const uint32_t *t_sorted, uint64_t n, uint32_t *iters);
/* Lloyd's k-means with k = 2 from k-means++ seeds (reading R27): c1 a uniform
 * row, c2 a row drawn with D^2 weights, both from Philox4x32-10 on the counter
 * (t[0], t[n-1], n, 0x4B4D5050) and key seed; returns the cut (0: none) and
 * the seeds *c1, *c2 (either pointer may be NULL). */
uint64_t or_kmpp_cut(const uint32_t *t_sorted, uint64_t n, uint64_t seed, uint32_t *c1, uint32_t *c2,
                     uint32_t *iters);
/* Exact optimal 1-D k-means of sorted t[0..n) ("k-means ... any number
 * above 2", reading R29): the partition into min(k, #distinct values) groups of
 * consecutive distinct values with the least total SSE; among optimal ones the
 * one whose last cut is smallest, then the cut before it, and so on.  Writes
 * the cuts (row indices, ascending) to cuts[0 .. groups-2] and returns the
 * number of groups (0 when n < 2 or all values are equal). */
uint32_t or_kmeans_cuts(const uint32_t *t_sorted, uint64_t n, uint32_t k, uint64_t *cuts);
/* Eq. 3: m = ceil((V/S^2) * (z/eps)^2) for a cluster with moments. */
double or_eq3_m(uint64_t n, uint64_t S, uint64_t Q_lo, uint64_t Q_hi, double eps, double z, int clamp);
/* Eq. 6, corrected numerator: k clusters given a_i = mu_i, b_i = V_i
 * (as doubles), total T; writes m[i] (ceil, clamped to >= 1). */
void or_eq6_m(uint32_t k, const double *mu, const double *V, double T, double eps, double z, double *m_out);
/* ROOT decision on one cluster [0, n) of sorted t: returns 1 if the split at
 * or_best_cut is accepted (Eq. 7 vs Eq. 8). tau_old/tau_new out. */
int  or_root_decide(const uint32_t *t_sorted, uint64_t n, double eps, double z, int clamp,
                    double *tau_old, double *tau_new, uint64_t *cut);
/* Exact sum of non-negative doubles, rounded once to nearest. */
double or_exact_sum(const double *x, uint64_t n);
/* Exact sum of finite doubles of either sign, rounded once to nearest. */
double or_exact_sum_signed(const double *x, uint64_t n);
/* Correctly rounded u128 -> double. */
double or_u128_to_double(uint64_t lo, uint64_t hi);
/* Inverse standard normal (AS241 PPND16); z for two-sided confidence conf. */
double or_z_from_conf(double conf);

#ifdef __cplusplus
}
#endif
#endif
