/*
 * stemroot_oracle.c -- TEST INFRASTRUCTURE ONLY (see stemroot_oracle.h).
 *
 * A plain, slow, single-threaded implementation of the STEM+ROOT sampling
 * plan, in the order of PAPER.md §3 and the normative algorithm recorded in
 * DESIGN.md §3 ("Readings").  Build: gcc -O2 -std=c11 -ffp-contract=off.
 * Every fp64 expression is written in the order DESIGN.md fixes, and
 * -ffp-contract=off keeps gcc from fusing a*b+c into an FMA.
 *
 * It shares no code with the CUDA library.  Nothing in the product path may
 * load this file.
 */
#include "stemroot_oracle.h"

#include <math.h>
#include <stdlib.h>
#include <string.h>

typedef unsigned __int128 u128;
typedef __int128 i128;

/* ------------------------------------------------------------------------ */
/* Exact integer helpers                                                     */
/* ------------------------------------------------------------------------ */

/* Correctly rounded conversion of a 128-bit unsigned integer to double.
 * gcc's (double)(unsigned __int128) is exact-then-round-to-nearest. */
static double rn128(u128 v) { return (double)v; }
static double rn64(uint64_t v) { return (double)v; }

double or_u128_to_double(uint64_t lo, uint64_t hi) {
    return rn128(((u128)hi << 64) | lo);
}

/* schoolbook multiply of little-endian 64-bit limb arrays: out[na+nb] */
static void limb_mul(const uint64_t *a, int na, const uint64_t *b, int nb, uint64_t *out) {
    for (int i = 0; i < na + nb; i++) out[i] = 0;
    for (int i = 0; i < na; i++) {
        uint64_t carry = 0;
        for (int j = 0; j < nb; j++) {
            u128 cur = (u128)a[i] * b[j] + out[i + j] + carry;
            out[i + j] = (uint64_t)cur;
            carry = (uint64_t)(cur >> 64);
        }
        out[i + nb] = carry;
    }
}

/* compare little-endian limb arrays of equal length: -1, 0, +1 */
static int limb_cmp(const uint64_t *a, const uint64_t *b, int n) {
    for (int i = n - 1; i >= 0; i--) {
        if (a[i] != b[i]) return a[i] < b[i] ? -1 : 1;
    }
    return 0;
}

/* Split-score comparison for the 2-means cut (R5):
 * score(k) = D_k^2 / p_k with D_k = n*S_L(k) - S*k, p_k = k*(n-k).
 * Compare D_a^2 * p_b against D_b^2 * p_a exactly (|D| < 2^96, p < 2^64:
 * both products < 2^256).  Returns -1/0/+1 for score_a <,=,> score_b. */
static int score_cmp(u128 absDa, uint64_t pa, u128 absDb, uint64_t pb) {
    uint64_t da[2] = {(uint64_t)absDa, (uint64_t)(absDa >> 64)};
    uint64_t db[2] = {(uint64_t)absDb, (uint64_t)(absDb >> 64)};
    uint64_t da2[4], db2[4], lhs[5], rhs[5];
    limb_mul(da, 2, da, 2, da2);
    limb_mul(db, 2, db, 2, db2);
    limb_mul(da2, 4, &pb, 1, lhs);
    limb_mul(db2, 4, &pa, 1, rhs);
    return limb_cmp(lhs, rhs, 5);
}

/* ------------------------------------------------------------------------ */
/* Exact sum of non-negative doubles (R12)                          */
/* A fixed-point accumulator of 32-bit digits; value = acc * 2^-OR_FIX_LSB.   */
/* ------------------------------------------------------------------------ */
#define OR_FIX_LSB 1100            /* covers every positive double's LSB (>= 2^-1074) */
#define OR_FIX_DIGITS 72           /* 72*32 = 2304 bits: 2^-1100 .. 2^1204            */

typedef struct { uint32_t d[OR_FIX_DIGITS]; } fixacc;

static void fix_add(fixacc *acc, double x) {
    if (!(x > 0.0)) return;                 /* zero contributes nothing */
    int e;
    double fr = frexp(x, &e);               /* x = fr * 2^e, fr in [0.5,1) */
    uint64_t mant = (uint64_t)ldexp(fr, 53);/* exact 53-bit integer       */
    int shift = e - 53 + OR_FIX_LSB;        /* x = mant * 2^(e-53)        */
    /* add mant << shift, 32 bits at a time, propagating carries */
    int digit = shift / 32, off = shift % 32;
    u128 v = (u128)mant << off;             /* at most 53+31 = 84 bits    */
    uint64_t carry = 0;
    for (int i = digit; i < OR_FIX_DIGITS; i++) {
        uint64_t add = (uint64_t)(v & 0xffffffffu);
        v >>= 32;
        uint64_t s = (uint64_t)acc->d[i] + add + carry;
        acc->d[i] = (uint32_t)s;
        carry = s >> 32;
        if (v == 0 && carry == 0) break;
    }
}

/* round-to-nearest-even of the accumulator to double */
static double fix_round(const fixacc *acc) {
    int top = -1;
    for (int i = OR_FIX_DIGITS - 1; i >= 0; i--) if (acc->d[i]) { top = i; break; }
    if (top < 0) return 0.0;
    int msb = top * 32 + (31 - __builtin_clz(acc->d[top]));   /* bit index of MSB */
    /* collect bits [msb-63, msb] into a 64-bit word, sticky-OR the rest */
    int lo_bit = msb - 63;
    uint64_t word = 0;
    int sticky = 0;
    for (int b = msb; b >= 0; b--) {
        int bit = (acc->d[b / 32] >> (b % 32)) & 1;
        if (b >= lo_bit) word = (word << 1) | (uint64_t)bit;
        else if (bit) { sticky = 1; break; }
    }
    if (lo_bit < 0) lo_bit = 0;   /* fewer than 64 significant bits: word is exact */
    word |= (uint64_t)sticky;   /* 11 guard bits below the 53 kept: sticky is enough */
    return ldexp(rn64(word), lo_bit - OR_FIX_LSB);
}

double or_exact_sum(const double *x, uint64_t n) {
    fixacc *acc = calloc(1, sizeof(fixacc));
    if (!acc) return NAN;
    for (uint64_t i = 0; i < n; i++) fix_add(acc, x[i]);
    double r = fix_round(acc);
    free(acc);
    return r;
}

/* Signed exact sum: positive and negative terms in two accumulators, the exact
 * difference |pos - neg| formed digit by digit, rounded once. */
typedef struct { fixacc pos, neg; } sfixacc;

static void sfix_add(sfixacc *a, double x) {
    if (x > 0.0) fix_add(&a->pos, x);
    else if (x < 0.0) fix_add(&a->neg, -x);
}

static double sfix_round(const sfixacc *a) {
    int cmp = 0;
    for (int i = OR_FIX_DIGITS - 1; i >= 0 && !cmp; i--)
        if (a->pos.d[i] != a->neg.d[i]) cmp = a->pos.d[i] > a->neg.d[i] ? 1 : -1;
    if (cmp == 0) return 0.0;
    const fixacc *big = cmp > 0 ? &a->pos : &a->neg, *small = cmp > 0 ? &a->neg : &a->pos;
    fixacc diff;
    int64_t borrow = 0;
    for (int i = 0; i < OR_FIX_DIGITS; i++) {
        int64_t d = (int64_t)big->d[i] - (int64_t)small->d[i] - borrow;
        borrow = d < 0;
        diff.d[i] = (uint32_t)(d + (borrow ? ((int64_t)1 << 32) : 0));
    }
    double r = fix_round(&diff);
    return cmp > 0 ? r : -r;
}

double or_exact_sum_signed(const double *x, uint64_t n) {
    sfixacc *acc = calloc(1, sizeof(sfixacc));
    if (!acc) return NAN;
    for (uint64_t i = 0; i < n; i++) sfix_add(acc, x[i]);
    double r = sfix_round(acc);
    free(acc);
    return r;
}

/* ------------------------------------------------------------------------ */
/* Philox4x32-10 (Random123), used for sampling with replacement    */
/* ------------------------------------------------------------------------ */
void or_philox4x32_10(const uint32_t ctr[4], const uint32_t key[2], uint32_t out[4]) {
    uint32_t x0 = ctr[0], x1 = ctr[1], x2 = ctr[2], x3 = ctr[3];
    uint32_t k0 = key[0], k1 = key[1];
    for (int round = 0; round < 10; round++) {
        uint64_t p0 = (uint64_t)0xD2511F53u * x0;
        uint64_t p1 = (uint64_t)0xCD9E8D57u * x2;
        uint32_t y0 = (uint32_t)(p1 >> 32) ^ x1 ^ k0;
        uint32_t y1 = (uint32_t)p1;
        uint32_t y2 = (uint32_t)(p0 >> 32) ^ x3 ^ k1;
        uint32_t y3 = (uint32_t)p0;
        x0 = y0; x1 = y1; x2 = y2; x3 = y3;
        k0 += 0x9E3779B9u;
        k1 += 0xBB67AE85u;
    }
    out[0] = x0; out[1] = x1; out[2] = x2; out[3] = x3;
}

/* ------------------------------------------------------------------------ */
/* Inverse normal: AS241 (Wichura 1988) PPND16                               */
/* ------------------------------------------------------------------------ */
static double ppnd16(double p) {
    double q = p - 0.5, r, val;
    if (fabs(q) <= 0.425) {
        r = 0.180625 - q * q;
        val = q * (((((((2.5090809287301226727e+3 * r + 3.3430575583588128105e+4) * r +
                        6.7265770927008700853e+4) * r + 4.5921953931549871457e+4) * r +
                      1.3731693765509461125e+4) * r + 1.9715909503065514427e+3) * r +
                    1.3314166789178437745e+2) * r + 3.3871328727963666080e0) /
              (((((((5.2264952788528545610e+3 * r + 2.8729085735721942674e+4) * r +
                    3.9307895800092710610e+4) * r + 2.1213794301586595867e+4) * r +
                  5.3941960214247511077e+3) * r + 6.8718700749205790830e+2) * r +
                4.2313330701600911252e+1) * r + 1.0);
        return val;
    }
    r = (q < 0) ? p : 1.0 - p;
    r = sqrt(-log(r));
    if (r <= 5.0) {
        r -= 1.6;
        val = (((((((7.74545014278341407640e-4 * r + 2.27238449892691845833e-2) * r +
                    2.41780725177450611770e-1) * r + 1.27045825245236838258e0) * r +
                  3.64784832476320460504e0) * r + 5.76949722146069140550e0) * r +
                4.63033784615654529590e0) * r + 1.42343711074968357734e0) /
              (((((((1.05075007164441684324e-9 * r + 5.47593808499534494600e-4) * r +
                    1.51986665636164571966e-2) * r + 1.48103976427480074590e-1) * r +
                  6.89767334985100004550e-1) * r + 1.67638483018380384940e0) * r +
                2.05319162663775882187e0) * r + 1.0);
    } else {
        r -= 5.0;
        val = (((((((2.01033439929228813265e-7 * r + 2.71155556874348757815e-5) * r +
                    1.24266094738807843860e-3) * r + 2.65321895265761230930e-2) * r +
                  2.96560571828504891230e-1) * r + 1.78482653991729133580e0) * r +
                5.46378491116411436990e0) * r + 6.65790464350110377720e0) /
              (((((((2.04426310338993978564e-15 * r + 1.42151175831644588870e-7) * r +
                    1.84631831751005468180e-5) * r + 7.86869131145613259100e-4) * r +
                  1.48753612908506148525e-2) * r + 1.36929880922735805310e-1) * r +
                5.99832206555887937690e-1) * r + 1.0);
    }
    return (q < 0.0) ? -val : val;
}

/* Two-sided z for confidence 1 - alpha: z = Phi^-1(1 - alpha/2). */
double or_z_from_conf(double conf) {
    if (!(conf > 0.0 && conf < 1.0)) return NAN;
    return ppnd16(1.0 - (1.0 - conf) / 2.0);
}

/* ------------------------------------------------------------------------ */
/* Cluster moments over a sorted range (n, S = sum t, Q = sum t^2)           */
/* ------------------------------------------------------------------------ */
typedef struct { uint64_t n, S; u128 Q; } moments;

static moments range_moments(const uint32_t *t, uint64_t lo, uint64_t hi) {
    moments m = {hi - lo, 0, 0};
    for (uint64_t i = lo; i < hi; i++) {
        m.S += t[i];
        m.Q += (u128)t[i] * t[i];
    }
    return m;
}

/* V = n*Q - S^2 = n^2 sigma^2 (population sigma, R3) */
static u128 moments_V(moments m) { return (u128)m.n * m.Q - (u128)m.S * m.S; }

/* ------------------------------------------------------------------------ */
/* ROOT sub-clustering: exact optimal 1-D 2-means (R5)        */
/* ------------------------------------------------------------------------ */
/* Cut k in [1, n-1] places t[lo..lo+k) left, t[lo+k..hi) right.  Only cuts
 * between distinct values are candidates.  Maximises D^2/(k(n-k)) exactly;
 * ties go to the smallest k.  Returns 0 when no candidate exists. */
static uint64_t best_cut(const uint32_t *t, uint64_t lo, uint64_t hi, uint64_t S) {
    uint64_t n = hi - lo, best_k = 0, best_p = 0;
    u128 best_absD = 0;
    uint64_t SL = 0;
    for (uint64_t k = 1; k < n; k++) {
        SL += t[lo + k - 1];
        if (!(t[lo + k - 1] < t[lo + k])) continue;
        i128 D = (i128)((u128)n * SL) - (i128)((u128)S * k);
        u128 absD = D < 0 ? (u128)(-D) : (u128)D;
        uint64_t p = k * (n - k);
        if (best_k == 0 || score_cmp(absD, p, best_absD, best_p) > 0) {
            best_k = k; best_absD = absD; best_p = p;
        }
    }
    return best_k;
}

/* Lloyd's algorithm for k = 2 (reading R26), written as the
 * textbook iteration on the cluster's values:
 *   1. centroids c1 = min t, c2 = max t;
 *   2. assignment: a value goes to cluster 1 iff it is not farther from c1 than
 *      from c2, i.e. 2 t <= c1 + c2 (a tie at the midpoint goes to cluster 1);
 *   3. update: c1, c2 = the means of the two clusters;
 *   4. repeat 2-3 until the assignment no longer changes (at most
 *      OR_LLOYD_MAX_ITERS assignment steps).
 * Centroids are kept as exact fractions S_1/k and S_2/(n-k), so step 2 is the
 * integer test 2 t k (n-k) <= S_1 (n-k) + S_2 k.  Sorted values make every
 * assignment a cut: cluster 1 = t[lo .. lo+k).  Returns k (0: no cut, the
 * cluster is constant or has < 2 rows). */
#define OR_LLOYD_MAX_ITERS 1000
static uint64_t lloyd_from(const uint32_t *t, uint64_t lo, uint64_t hi, uint64_t mid2, uint32_t *iters);

static uint64_t lloyd_cut(const uint32_t *t, uint64_t lo, uint64_t hi, uint32_t *iters) {
    if (iters) *iters = 0;
    if (hi - lo < 2 || t[lo] == t[hi - 1]) return 0;
    /* step 1: centroids (min, max) */
    return lloyd_from(t, lo, hi, (uint64_t)t[lo] + t[hi - 1], iters);
}

/* k-means++ seeding for k = 2 (Arthur & Vassilvitskii's D^2 weighting; the
 * randomised initialisation of a library k-means, reading R27),
 * with the random numbers drawn from Philox4x32-10 (P10) on the counter
 * (min t, max t, n, 'KMPP') and the plan's seed as key:
 *   1. c1 = t[lo + j1], j1 = floor(u * n), u = (x1:x0) / 2^64 (uniform row);
 *   2. c2 = t[lo + j2], row j2 drawn with probability (t[lo+j2] - c1)^2 / W,
 *      W = sum_i (t_i - c1)^2: j2 = the first row whose running sum of
 *      (t_i - c1)^2 exceeds R = floor(W x2 / 2^32).
 * Then Lloyd's steps 2-4 as above from the centroids (c1, c2).  Returns the cut
 * k (0 for a constant cluster or < 2 rows); c1, c2 are reported when asked. */
static uint64_t kmpp_cut(const uint32_t *t, uint64_t lo, uint64_t hi, uint64_t seed, uint32_t *c1o,
                         uint32_t *c2o, uint32_t *iters) {
    uint64_t n = hi - lo;
    if (iters) *iters = 0;
    if (n < 2 || t[lo] == t[hi - 1]) return 0;
    const uint32_t ctr[4] = {t[lo], t[hi - 1], (uint32_t)n, 0x4B4D5050u};
    const uint32_t key[2] = {(uint32_t)seed, (uint32_t)(seed >> 32)};
    uint32_t x[4];
    or_philox4x32_10(ctr, key, x);
    uint64_t j1 = (uint64_t)(((u128)((((uint64_t)x[1]) << 32) | x[0]) * n) >> 64);
    uint32_t c1 = t[lo + j1];
    u128 W = 0;
    for (uint64_t i = lo; i < hi; i++) {
        uint64_t d = t[i] > c1 ? (uint64_t)t[i] - c1 : (uint64_t)c1 - t[i];
        W += (u128)d * d;
    }
    u128 R = (W * x[2]) >> 32;
    u128 run = 0;
    uint64_t j2 = 0;
    for (uint64_t i = lo; i < hi; i++) {
        uint64_t d = t[i] > c1 ? (uint64_t)t[i] - c1 : (uint64_t)c1 - t[i];
        run += (u128)d * d;
        if (run > R) { j2 = i - lo; break; }
    }
    uint32_t c2 = t[lo + j2];
    if (c1o) *c1o = c1;
    if (c2o) *c2o = c2;
    return lloyd_from(t, lo, hi, (uint64_t)c1 + c2, iters);
}

/* Lloyd's steps 2-4 from centroids whose sum is mid2 (both centroids are
 * values of the cluster, distinct, so the first cut is in [1, n)). */
static uint64_t lloyd_from(const uint32_t *t, uint64_t lo, uint64_t hi, uint64_t mid2, uint32_t *iters) {
    uint64_t n = hi - lo;
    uint64_t k = 0;
    for (uint64_t i = lo; i < hi; i++)
        if (2 * (uint64_t)t[i] <= mid2) k++;
    uint32_t it = 1;
    for (; it < OR_LLOYD_MAX_ITERS; it++) {
        /* step 3: exact centroid sums of the current assignment */
        uint64_t S1 = 0, S2 = 0;
        for (uint64_t i = lo; i < lo + k; i++) S1 += t[i];
        for (uint64_t i = lo + k; i < hi; i++) S2 += t[i];
        /* step 2 with the new centroids */
        const u128 rhs = (u128)S1 * (n - k) + (u128)S2 * k;
        const u128 f = (u128)2 * k * (n - k);
        uint64_t k2 = 0;
        for (uint64_t i = lo; i < hi; i++)
            if ((u128)t[i] * f <= rhs) k2++;
        if (k2 == k) break;
        k = k2;
    }
    if (iters) *iters = it;
    return k;
}

uint64_t or_lloyd_cut(const uint32_t *t_sorted, uint64_t n, uint32_t *iters) {
    return lloyd_cut(t_sorted, 0, n, iters);
}

uint64_t or_kmpp_cut(const uint32_t *t_sorted, uint64_t n, uint64_t seed, uint32_t *c1, uint32_t *c2,
                     uint32_t *iters) {
    return kmpp_cut(t_sorted, 0, n, seed, c1, c2, iters);
}

uint64_t or_best_cut(const uint32_t *t_sorted, uint64_t n) {
    if (n < 2) return 0;
    moments m = range_moments(t_sorted, 0, n);
    return best_cut(t_sorted, 0, n, m.S);
}

/* ------------------------------------------------------------------------ */
/* Exact optimal 1-D k-means (split = 3; "k-means ... any number above */
/* 2 works well"; reading R29)                                                */
/* ------------------------------------------------------------------------ */
/* Total SSE of a partition = Q - sum_g S_g^2 / n_g, so the optimal partition
 * maximises sum_g S_g^2 / n_g.  In 1-D some optimal partition consists of
 * consecutive sorted values and never separates equal values, so the groups
 * are runs of consecutive distinct values and the textbook dynamic program
 *   F[1][b] = S(0,b)^2 / n(0,b),
 *   F[j][b] = max_{a < b} F[j-1][a] + S(a,b)^2 / n(a,b)
 * over the distinct values is exact.  Every F is kept as an exact fraction of
 * big integers (num / den, den = product of the group sizes), so comparisons
 * are exact; ties take the smallest a, i.e. among optimal partitions the one
 * whose last cut is smallest, then the one before it, and so on. */
#define OR_BIG 12          /* 768-bit: num * den' < 2^(96 + 64 k + 3) for k <= 8 */
typedef struct { uint64_t w[OR_BIG]; } bigint;
typedef struct { bigint num, den; } fraction;

static bigint big_mul(const bigint *a, const bigint *b) {
    uint64_t out[2 * OR_BIG];
    limb_mul(a->w, OR_BIG, b->w, OR_BIG, out);
    bigint r;
    memcpy(r.w, out, sizeof(r.w));   /* the high half is zero for k <= 8 */
    return r;
}

static bigint big_add(const bigint *a, const bigint *b) {
    bigint r;
    u128 carry = 0;
    for (int i = 0; i < OR_BIG; i++) {
        u128 s = (u128)a->w[i] + b->w[i] + carry;
        r.w[i] = (uint64_t)s;
        carry = s >> 64;
    }
    return r;
}

static bigint big_u128(u128 v) {
    bigint r;
    memset(&r, 0, sizeof(r));
    r.w[0] = (uint64_t)v;
    r.w[1] = (uint64_t)(v >> 64);
    return r;
}

/* f + S^2 / n */
static fraction frac_add_group(const fraction *f, uint64_t S, uint64_t n) {
    bigint bn = big_u128(n), s2 = big_u128((u128)S * S);
    bigint a = big_mul(&f->num, &bn), b = big_mul(&s2, &f->den);
    fraction r;
    r.num = big_add(&a, &b);
    r.den = big_mul(&f->den, &bn);
    return r;
}

static int frac_cmp(const fraction *a, const fraction *b) {
    bigint l = big_mul(&a->num, &b->den), r = big_mul(&b->num, &a->den);
    return limb_cmp(l.w, r.w, OR_BIG);
}

uint32_t or_kmeans_cuts(const uint32_t *t, uint64_t n, uint32_t k, uint64_t *cuts) {
    if (n < 2 || t[0] == t[n - 1] || k < 2) return 0;
    /* run starts of the distinct values: pos[0] = 0 < ... < pos[d-1], pos[d] = n */
    uint64_t d = 1;
    for (uint64_t i = 1; i < n; i++) d += t[i - 1] < t[i];
    uint64_t *pos = malloc((d + 1) * sizeof(uint64_t)), *P = malloc((d + 1) * sizeof(uint64_t));
    uint32_t K = k < d ? k : (uint32_t)d;
    fraction *F = malloc((size_t)(K + 1) * (d + 1) * sizeof(fraction));
    uint64_t *arg = malloc((size_t)(K + 1) * (d + 1) * sizeof(uint64_t));
    if (!pos || !P || !F || !arg) { free(pos); free(P); free(F); free(arg); return 0; }
    uint64_t r = 0, run = 0;
    for (uint64_t i = 0; i < n; i++) {
        if (i == 0 || t[i - 1] < t[i]) { pos[r] = i; P[r] = run; r++; }
        run += t[i];
    }
    pos[d] = n;
    P[d] = run;
#define FF(j, b) F[(size_t)(j) * (d + 1) + (b)]
#define ARG(j, b) arg[(size_t)(j) * (d + 1) + (b)]
    fraction zero;
    memset(&zero, 0, sizeof(zero));
    zero.den.w[0] = 1;
    for (uint64_t b = 1; b <= d; b++) FF(1, b) = frac_add_group(&zero, P[b], pos[b]);
    for (uint32_t j = 2; j <= K; j++)
        for (uint64_t b = j; b <= d; b++) {
            for (uint64_t a = j - 1; a < b; a++) {
                fraction c = frac_add_group(&FF(j - 1, a), P[b] - P[a], pos[b] - pos[a]);
                if (a == j - 1 || frac_cmp(&c, &FF(j, b)) > 0) {   /* strict: ties keep the smaller a */
                    FF(j, b) = c;
                    ARG(j, b) = a;
                }
            }
        }
    uint64_t b = d;
    for (uint32_t j = K; j >= 2; j--) {
        b = ARG(j, b);
        cuts[j - 2] = pos[b];
    }
#undef FF
#undef ARG
    free(pos); free(P); free(F); free(arg);
    return K;
}

/* ------------------------------------------------------------------------ */
/* STEM sample sizes                                                          */
/* ------------------------------------------------------------------------ */
/* Eq. 3 in the fixed order of R9: x = (rn(V)/(rn(S)*rn(S))) * k2,
 * k2 = (z/eps)^2, m = ceil(x), clamped to >= 1 when clamp. */
static double eq3_m(u128 V, uint64_t S, double k2, int clamp) {
    if (V == 0) return clamp ? 1.0 : 0.0;
    double x = (rn128(V) / (rn64(S) * rn64(S))) * k2;
    double m = ceil(x);
    if (clamp && m < 1.0) m = 1.0;
    return m;
}

double or_eq3_m(uint64_t n, uint64_t S, uint64_t Q_lo, uint64_t Q_hi, double eps, double z, int clamp) {
    moments m = {n, S, ((u128)Q_hi << 64) | Q_lo};
    double q = z / eps;
    return eq3_m(moments_V(m), S, q * q, clamp);
}

/* Eq. 6 with the numerator of the derivation (reading R1):
 * m_i = ceil( (sum_j sqrt(a_j b_j)) / c * sqrt(b_i / a_i) ),
 * a_i = mu_i, b_i = V_i, c = (eps * T / z)^2. */
static double eq6_one(double g, double mu, double V, int clamp) {
    if (V == 0.0) return clamp ? 1.0 : 0.0;
    double m = ceil(g * sqrt(V / mu));
    if (clamp && m < 1.0) m = 1.0;
    return m;
}

void or_eq6_m(uint32_t k, const double *mu, const double *V, double T, double eps, double z, double *m_out) {
    double w = (eps * T) / z;
    double c = w * w;
    double *terms = calloc(k ? k : 1, sizeof(double));
    for (uint32_t i = 0; i < k; i++) terms[i] = sqrt(mu[i] * V[i]);
    double ssum = or_exact_sum(terms, k);
    free(terms);
    double g = ssum / c;
    for (uint32_t i = 0; i < k; i++) m_out[i] = eq6_one(g, mu[i], V[i], 1);
}

/* ------------------------------------------------------------------------ */
/* ROOT decision (Eq. 7 vs Eq. 8; readings R6-R9)                */
/* ------------------------------------------------------------------------ */
#define OR_KMAX 8
typedef struct {
    double tau_old, tau_new;
    uint64_t cut;                 /* 2-way rules: the cut */
    uint32_t ngroups;             /* children if split (2, or 2..kmeans_k for split = 3) */
    uint64_t cuts[OR_KMAX - 1];   /* their boundaries, relative to lo, ascending */
    int split;
} decision;

/* Eq. 8 for the children [lo + b_{g-1}, lo + b_g) of a cluster, b_0 = 0 and
 * b_G = n, Eq. 6 (corrected numerator) over them with c from the parent's
 * total, summed left to right (for two children exactly the 2-way formula). */
static double tau_children(const uint32_t *t, uint64_t lo, uint64_t hi, const uint64_t *cuts, uint32_t G,
                           double eps, double z, int clamp, uint64_t S_parent) {
    double mu[OR_KMAX], V[OR_KMAX];
    for (uint32_t g = 0; g < G; g++) {
        uint64_t a = g == 0 ? lo : lo + cuts[g - 1], b = g + 1 == G ? hi : lo + cuts[g];
        moments m = range_moments(t, a, b);
        mu[g] = rn64(m.S) / rn64(m.n);
        V[g] = rn128(moments_V(m));
    }
    double w = (eps * rn64(S_parent)) / z;
    double c = w * w;
    double ssum = 0.0;
    for (uint32_t g = 0; g < G; g++) ssum = g == 0 ? sqrt(mu[0] * V[0]) : ssum + sqrt(mu[g] * V[g]);
    double gg = ssum / c;
    double tau = 0.0;
    for (uint32_t g = 0; g < G; g++) {
        double m = eq6_one(gg, mu[g], V[g], clamp);
        tau = g == 0 ? m * mu[0] : tau + m * mu[g];
    }
    return tau;
}

static decision root_decide(const uint32_t *t, uint64_t lo, uint64_t hi, double eps, double z,
                            double k2, int clamp, int split, uint64_t seed, uint32_t kk) {
    decision d;
    memset(&d, 0, sizeof(d));
    uint64_t n = hi - lo;
    if (n < 2 || t[lo] == t[hi - 1]) return d;              /* R5: leaf */
    moments all = range_moments(t, lo, hi);
    if (split == 3) {                                       /* R29: k groups at once */
        d.ngroups = or_kmeans_cuts(t + lo, n, kk, d.cuts);
        d.cut = d.cuts[0];
    } else {
        uint64_t k = split == 1   ? lloyd_cut(t, lo, hi, NULL)
                   : split == 2 ? kmpp_cut(t, lo, hi, seed, NULL, NULL, NULL)
                                : best_cut(t, lo, hi, all.S);
        d.cut = k;
        d.cuts[0] = k;
        d.ngroups = 2;
    }
    /* Eq. 7: tau_old = m * Xbar with m from Eq. 3 */
    double mu = rn64(all.S) / rn64(all.n);
    double m_old = eq3_m(moments_V(all), all.S, k2, clamp);
    d.tau_old = m_old * mu;
    /* Eq. 8: tau_new = sum_i m_i Xbar_i with m_i from Eq. 6 over the children */
    d.tau_new = tau_children(t, lo, hi, d.cuts, d.ngroups, eps, z, clamp, all.S);
    d.split = d.tau_new < d.tau_old;                        /* strict */
    return d;
}

int or_root_decide(const uint32_t *t_sorted, uint64_t n, double eps, double z, int clamp,
                   double *tau_old, double *tau_new, uint64_t *cut) {
    double q = z / eps;
    decision d = root_decide(t_sorted, 0, n, eps, z, q * q, clamp, 0, 0, 2);
    if (tau_old) *tau_old = d.tau_old;
    if (tau_new) *tau_new = d.tau_new;
    if (cut) *cut = d.cut;
    return d.split;
}

/* ------------------------------------------------------------------------ */
/* Whole plan                                                                 */
/* ------------------------------------------------------------------------ */
typedef struct { uint32_t kid, t, row; } trow;

static int trow_cmp(const void *a, const void *b) {
    const trow *x = a, *y = b;
    if (x->kid != y->kid) return x->kid < y->kid ? -1 : 1;
    if (x->t != y->t) return x->t < y->t ? -1 : 1;
    if (x->row != y->row) return x->row < y->row ? -1 : 1;
    return 0;
}

typedef struct { uint32_t kid; uint64_t lo, hi; } leaf;
typedef struct { leaf *v; uint64_t n, cap; } leafvec;

static int leaf_push(leafvec *lv, leaf x) {
    if (lv->n == lv->cap) {
        uint64_t nc = lv->cap ? lv->cap * 2 : 1024;
        leaf *nv = realloc(lv->v, nc * sizeof(leaf));
        if (!nv) return -1;
        lv->v = nv; lv->cap = nc;
    }
    lv->v[lv->n++] = x;
    return 0;
}

typedef struct { uint64_t lo, hi; uint32_t depth; } work_item;
typedef struct { work_item *v; uint64_t n, cap; } workvec;

static int work_push(workvec *wv, uint64_t lo, uint64_t hi, uint32_t depth) {
    if (wv->n == wv->cap) {
        uint64_t nc = wv->cap ? wv->cap * 2 : 256;
        work_item *nv = realloc(wv->v, nc * sizeof(work_item));
        if (!nv) return -1;
        wv->v = nv; wv->cap = nc;
    }
    work_item w = {lo, hi, depth};
    wv->v[wv->n++] = w;
    return 0;
}

void or_plan_free(or_plan *p) {
    if (!p) return;
    free(p->kernel_id); free(p->ordinal); free(p->lo_ns); free(p->hi_ns);
    free(p->n); free(p->sum_ns); free(p->m); free(p->mean_ns); free(p->std_ns);
    free(p->census); free(p->sample_row); free(p->sample_cluster); free(p->sample_weight);
    free(p->est_metric); free(p->true_metric); free(p->bound_metric);
    free(p);
}

int or_plan_build(uint64_t n, uint32_t n_kernels, const uint32_t *kernel_id,
                  const uint32_t *exec_ns, uint32_t n_metrics, const double *metrics,
                  double eps, const or_opts *opts, or_plan **out) {
    if (!out) return OR_E_INVAL;
    *out = NULL;
    if (!opts || !kernel_id || !exec_ns || n == 0) return OR_E_INVAL;
    if (!(eps > 0.0 && eps < 1.0) || !(opts->z > 0.0) || !isfinite(opts->z)) return OR_E_INVAL;
    if (n_metrics > 64 || (n_metrics > 0 && !metrics)) return OR_E_INVAL;
    if (opts->scope < 0 || opts->scope > 2) return OR_E_INVAL;
    if (opts->split < 0 || opts->split > 3) return OR_E_INVAL;
    if (opts->split == 3 && (opts->kmeans_k < 2 || opts->kmeans_k > OR_KMAX)) return OR_E_INVAL;
    if (n >= ((uint64_t)1 << 32)) return OR_E_RANGE;
    for (uint64_t i = 0; i < n; i++) if (kernel_id[i] >= n_kernels) return OR_E_RANGE;

    const double z = opts->z;
    const double q = z / eps;
    const double k2 = q * q;
    const int clamp = opts->clamp_in_split ? 1 : 0;
    int status = OR_OK;

    /* Step 1: group by kernel: stable sort by (kernel_id, t), row breaks ties */
    trow *rows = malloc(n * sizeof(trow));
    uint32_t *t = malloc(n * sizeof(uint32_t));
    uint32_t *row_of = malloc(n * sizeof(uint32_t));
    leafvec leaves = {0, 0, 0};
    workvec work = {0, 0, 0};
    u128 *V = NULL;
    double *mu = NULL, *mreal = NULL, *terms = NULL;
    or_plan *p = calloc(1, sizeof(or_plan));
    if (!rows || !t || !row_of || !p) { status = OR_E_NOMEM; goto fail; }
    for (uint64_t i = 0; i < n; i++) {
        rows[i].kid = kernel_id[i]; rows[i].t = exec_ns[i]; rows[i].row = (uint32_t)i;
    }
    qsort(rows, n, sizeof(trow), trow_cmp);
    for (uint64_t i = 0; i < n; i++) { t[i] = rows[i].t; row_of[i] = rows[i].row; }

    /* Step 2: ROOT on each group, depth-first, left before right,
     * so leaves come out in canonical (kernel_id, lo) order. */
    uint32_t max_depth = 0;
    for (uint64_t g0 = 0; g0 < n;) {
        uint64_t g1 = g0;
        while (g1 < n && rows[g1].kid == rows[g0].kid) g1++;
        uint32_t kid = rows[g0].kid;
        if (work_push(&work, g0, g1, 0)) { status = OR_E_NOMEM; goto fail; }
        while (work.n > 0) {
            work_item w = work.v[--work.n];
            if (w.depth > max_depth) max_depth = w.depth;
            decision d;
            memset(&d, 0, sizeof(d));
            if (opts->root)
                d = root_decide(t, w.lo, w.hi, eps, z, k2, clamp, opts->split, opts->seed, (uint32_t)opts->kmeans_k);
            if (d.split) {
                /* push the children right to left: the leftmost is visited first */
                for (uint32_t g = d.ngroups; g-- > 0;) {
                    uint64_t a = g == 0 ? w.lo : w.lo + d.cuts[g - 1], b = g + 1 == d.ngroups ? w.hi : w.lo + d.cuts[g];
                    if (work_push(&work, a, b, w.depth + 1)) { status = OR_E_NOMEM; goto fail; }
                }
            } else {
                leaf lf = {kid, w.lo, w.hi};
                if (leaf_push(&leaves, lf)) { status = OR_E_NOMEM; goto fail; }
            }
        }
        g0 = g1;
    }
    p->max_depth = max_depth;

    /* Leaf statistics (Fig. 6) */
    uint64_t L = leaves.n;
    p->n_clusters = L;
    p->kernel_id = malloc(L * 4); p->ordinal = malloc(L * 4);
    p->lo_ns = malloc(L * 4); p->hi_ns = malloc(L * 4);
    p->n = malloc(L * 8); p->sum_ns = malloc(L * 8); p->m = malloc(L * 8);
    p->mean_ns = malloc(L * 8); p->std_ns = malloc(L * 8); p->census = calloc(L, 1);
    V = malloc(L * sizeof(u128));
    mu = malloc(L * 8); mreal = malloc(L * 8); terms = malloc(L * 8);
    if (!p->kernel_id || !p->ordinal || !p->lo_ns || !p->hi_ns || !p->n || !p->sum_ns ||
        !p->m || !p->mean_ns || !p->std_ns || !p->census || !V || !mu || !mreal || !terms) {
        status = OR_E_NOMEM; goto fail_leaves;
    }
    uint64_t T = 0;
    for (uint64_t i = 0; i < L; i++) {
        leaf lf = leaves.v[i];
        moments m = range_moments(t, lf.lo, lf.hi);
        p->kernel_id[i] = lf.kid;
        p->ordinal[i] = (i > 0 && leaves.v[i - 1].kid == lf.kid) ? p->ordinal[i - 1] + 1 : 0;
        p->lo_ns[i] = t[lf.lo];
        p->hi_ns[i] = t[lf.hi - 1];
        p->n[i] = m.n;
        p->sum_ns[i] = m.S;
        V[i] = moments_V(m);
        mu[i] = rn64(m.S) / rn64(m.n);
        p->mean_ns[i] = mu[i];
        p->std_ns[i] = sqrt(rn128(V[i])) / rn64(m.n);
        T += m.S;
    }

    /* Step 3: STEM sample sizes (Eq. 6 corrected, P:L169 + P:L464; R1, R10, R11) */
    if (opts->scope == 2) {
        for (uint64_t i = 0; i < L; i++) mreal[i] = eq3_m(V[i], p->sum_ns[i], k2, 1);
        p->ssum = NAN;
    } else {
        /* scope 0: one set = all leaves; scope 1: one set per kernel */
        uint64_t a = 0;
        while (a < L) {
            uint64_t b = a;
            if (opts->scope == 0) b = L;
            else while (b < L && p->kernel_id[b] == p->kernel_id[a]) b++;
            uint64_t Tset = 0;
            for (uint64_t i = a; i < b; i++) {
                Tset += p->sum_ns[i];
                terms[i - a] = sqrt(mu[i] * rn128(V[i]));
            }
            double ssum = or_exact_sum(terms, b - a);
            double w = (eps * rn64(Tset)) / z;
            double c = w * w;
            double g = ssum / c;
            for (uint64_t i = a; i < b; i++) mreal[i] = eq6_one(g, mu[i], rn128(V[i]), 1);
            if (opts->scope == 0) p->ssum = ssum;
            a = b;
        }
        if (opts->scope == 1) p->ssum = NAN;
    }
    uint64_t total_m = 0;
    for (uint64_t i = 0; i < L; i++) {
        double mi = mreal[i];
        if (opts->census_cap && mi >= rn64(p->n[i])) { mi = rn64(p->n[i]); p->census[i] = 1; }
        if (!(mi < 4294967296.0)) { status = OR_E_LIMIT; goto fail_leaves; }
        p->m[i] = (uint64_t)mi;
        total_m += p->m[i];
        if (total_m >= ((uint64_t)1 << 32)) { status = OR_E_LIMIT; goto fail_leaves; }
    }

    /* Step 4: random sampling with replacement (R14) */
    p->n_samples = total_m;
    p->sample_row = malloc((total_m ? total_m : 1) * 4);
    p->sample_cluster = malloc((total_m ? total_m : 1) * 4);
    p->sample_weight = malloc((total_m ? total_m : 1) * 8);
    p->n_metrics = n_metrics;
    p->est_metric = calloc(n_metrics ? n_metrics : 1, 8);
    if (!p->sample_row || !p->sample_cluster || !p->sample_weight || !p->est_metric) {
        status = OR_E_NOMEM; goto fail_leaves;
    }
    const uint32_t key[2] = {(uint32_t)opts->seed, (uint32_t)(opts->seed >> 32)};
    uint64_t s = 0;
    u128 sum_q = 0;
    double sum_frac = 0.0, sum_var = 0.0;
    for (uint64_t i = 0; i < L; i++) {
        leaf lf = leaves.v[i];
        uint64_t ni = p->n[i], mi = p->m[i];
        uint64_t U = 0;
        double wgt = rn64(ni) / rn64(mi);
        for (uint64_t j = 0; j < mi; j++) {
            uint64_t pos;
            if (p->census[i]) {
                pos = lf.lo + j;
            } else {
                uint32_t ctr[4] = {(uint32_t)(j >> 1), p->ordinal[i], p->kernel_id[i], 0x53544D31u};
                uint32_t x[4];
                or_philox4x32_10(ctr, key, x);
                uint64_t r = (j & 1) ? (((uint64_t)x[3] << 32) | x[2]) : (((uint64_t)x[1] << 32) | x[0]);
                pos = lf.lo + (uint64_t)(((u128)r * ni) >> 64);
            }
            p->sample_row[s] = row_of[pos];
            p->sample_cluster[s] = (uint32_t)i;
            p->sample_weight[s] = wgt;
            U += t[pos];
            for (uint32_t c = 0; c < n_metrics; c++)
                p->est_metric[c] += wgt * metrics[(uint64_t)c * n + row_of[pos]];
            s++;
        }
        /* Step 5: extrapolation: t_i = N_i * mean of samples */
        u128 num = (u128)ni * U;
        sum_q += num / mi;
        sum_frac += rn128(num % mi) / rn64(mi);
        sum_var += rn128(V[i]) / rn64(mi);
    }
    p->est_total_ns = rn128(sum_q) + sum_frac;
    p->true_total_ns = T;
    /* predicted bound, Eq. 5 / Eq. 12: z * sqrt(sum V_i/m_i) / T */
    p->bound = (T == 0) ? 0.0 : z * sqrt(sum_var) / rn64(T);
    p->eps = eps;
    p->z = z;

    /* Step 6 (metric_bounds, reading R28): the true total of each metric column
     * and its predicted relative error, Eq. 5 with the metric in place of the
     * time: bound_c = z sqrt(sum_i V_ic / m_i) / |true_c|,
     * V_ic = n_i^2 sigma_ic^2 = n_i * sum_j (x_j - xbar_ic)^2 over the leaf's rows
     * (population variance, R3), xbar_ic = (exact sum_j x_j) / n_i. */
    if (opts->metric_bounds && n_metrics) {
        p->true_metric = calloc(n_metrics, 8);
        p->bound_metric = calloc(n_metrics, 8);
        sfixacc *acc = malloc(sizeof(sfixacc));
        if (!p->true_metric || !p->bound_metric || !acc) { free(acc); status = OR_E_NOMEM; goto fail_leaves; }
        for (uint32_t c = 0; c < n_metrics; c++) {
            const double *col = metrics + (uint64_t)c * n;
            p->true_metric[c] = or_exact_sum_signed(col, n);
            double var_c = 0.0;
            for (uint64_t i = 0; i < L; i++) {
                leaf lf = leaves.v[i];
                memset(acc, 0, sizeof(sfixacc));
                for (uint64_t pos = lf.lo; pos < lf.hi; pos++) sfix_add(acc, col[row_of[pos]]);
                const double xbar = sfix_round(acc) / rn64(p->n[i]);
                memset(acc, 0, sizeof(sfixacc));
                for (uint64_t pos = lf.lo; pos < lf.hi; pos++) {
                    const double d = col[row_of[pos]] - xbar;
                    fix_add(&acc->pos, d * d);
                }
                const double Vc = rn64(p->n[i]) * fix_round(&acc->pos);
                var_c += Vc / rn64(p->m[i]);
            }
            const double tc = fabs(p->true_metric[c]);
            p->bound_metric[c] = tc > 0.0 ? z * sqrt(var_c) / tc : (var_c > 0.0 ? INFINITY : 0.0);
        }
        free(acc);
    }

    free(V); free(mu); free(mreal); free(terms);
    free(work.v); free(leaves.v); free(rows); free(t); free(row_of);
    *out = p;
    return OR_OK;

fail_leaves:
    free(V); free(mu); free(mreal); free(terms);
fail:
    free(work.v); free(leaves.v); free(rows); free(t); free(row_of);
    or_plan_free(p);
    return status;
}
