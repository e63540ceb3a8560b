// capi.cu -- the C ABI (include/stemroot.h): validation, workspace, stage
// orchestration on one stream, host plan assembly.  All arithmetic of the
// plan runs in the stage kernels (sort.cu, root.cu, stem.cu).
#include <cmath>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <new>
#include <utility>

#include "internal.h"

namespace sr {

cudaError_t &last_cuda_error() {
    static thread_local cudaError_t e = cudaSuccess;
    return e;
}

int Ctx::ensure_all(uint64_t n, uint32_t K, uint32_t n_metrics) {
    (void)n_metrics;
    CKS(ensure(keys[0], cap_keys[0], sizeof(uint64_t) * n));
    CKS(ensure(keys[1], cap_keys[1], sizeof(uint64_t) * n));
    CKS(ensure(vals[0], cap_vals[0], sizeof(uint32_t) * n));
    CKS(ensure(vals[1], cap_vals[1], sizeof(uint32_t) * n));
    CKS(ensure(t_sorted, cap_ts, sizeof(uint32_t) * (n + 4)));   // + slack: uint4 reads of the last rows
    CKS(ensure(row_sorted, cap_rs, sizeof(uint32_t) * (n + 1)));
    CKS(ensure(kid_count, cap_kc, sizeof(uint32_t) * ((uint64_t)K + 1)));
    CKS(ensure(goff, cap_goff, sizeof(uint32_t) * ((uint64_t)K + 2)));
    CKS(ensure(kid_max, cap_kmax, sizeof(uint32_t) * ((uint64_t)K + 1)));
    CKS(ensure(key_base, cap_kbase, sizeof(uint64_t) * ((uint64_t)K + 2)));
    CKS(ensure(key_base_c, cap_kbase_c, sizeof(uint64_t) * ((uint64_t)K + 2)));
    CKS(ensure(hist, cap_hist, sizeof(uint64_t) * 9 * 256));
    CKS(ensure(sort_mode, cap_sort_mode, sizeof(uint32_t) * 8));
    CKS(ensure(sort_gbase, cap_sort_gbase, sizeof(uint64_t) * 8 * 256));
    CKS(ensure(scalars, cap_scalars, sizeof(DevScalars)));
    CKS(ensure(scan_scratch, cap_scan, (scan_tiles((uint64_t)K + 2) + 1) * 32));
    CKS(ensure(PS1, cap_ps1, sizeof(uint64_t) * (n / kChunk + 2)));
    CKS(ensure(PS2, cap_ps2, sizeof(u128) * (n / kChunk + 2)));
    CKS(ensure(flags, cap_flags, sizeof(uint32_t) * (n / 32 + 4)));
    return STEM_OK;
}

template <class T>
static void dfree(T *&p, size_t &cap) {
    if (p) cudaFree(p);
    p = nullptr;
    cap = 0;
}

void Ctx::release() {
    plan_block_abort(*this);
    if (dstream) { cudaStreamDestroy(dstream); dstream = nullptr; }
    if (ev_pack) { cudaEventDestroy(ev_pack); ev_pack = nullptr; }
    if (ev_d2h) { cudaEventDestroy(ev_d2h); ev_d2h = nullptr; }
    for (auto &e : ev_h2d)
        if (e) { cudaEventDestroy(e); e = nullptr; }
    if (ev_pre) { cudaEventDestroy(ev_pre); ev_pre = nullptr; }
    if (ev_fork) cudaEventDestroy(ev_fork);
    if (ev_join) cudaEventDestroy(ev_join);
    if (side) cudaStreamDestroy(side);
    for (int i = 0; i < 4; i++)
        if (ev_lvl[i]) { cudaEventDestroy(ev_lvl[i]); ev_lvl[i] = nullptr; }
    if (h_lvl) { cudaFreeHost(h_lvl); h_lvl = nullptr; }
    for (int i = 0; i < 8; i++)
        if (ev_vr[i]) { cudaEventDestroy(ev_vr[i]); ev_vr[i] = nullptr; }
    if (h_vr) { cudaFreeHost(h_vr); h_vr = nullptr; }
    if (h_vcount) { cudaFreeHost(h_vcount); h_vcount = nullptr; }
    if (ev_vcount) { cudaEventDestroy(ev_vcount); ev_vcount = nullptr; }
    if (ev_vfork) cudaEventDestroy(ev_vfork);
    if (ev_vjoin) cudaEventDestroy(ev_vjoin);
    if (vside) cudaStreamDestroy(vside);
    ev_vfork = ev_vjoin = nullptr;
    vside = nullptr;
    ev_fork = ev_join = nullptr;
    side = nullptr;
    dfree(in_kid, cap_in_kid); dfree(in_t, cap_in_t); dfree(in_met, cap_in_met);
    for (int i = 0; i < 2; i++) {
        dfree(keys[i], cap_keys[i]); dfree(vals[i], cap_vals[i]);
        dfree(f_lo[i], cap_flo[i]); dfree(f_hi[i], cap_fhi[i]); dfree(f_aoff[i], cap_faoff[i]);
        dfree(f_S[i], cap_fS[i]); dfree(f_Q[i], cap_fQ[i]);
    }
    dfree(t_sorted, cap_ts); dfree(row_sorted, cap_rs); dfree(kid_count, cap_kc); dfree(goff, cap_goff);
    dfree(kid_max, cap_kmax); dfree(key_base, cap_kbase); dfree(key_base_c, cap_kbase_c); dfree(key_base_s, cap_kbase_s); dfree(tailh, cap_tailh); dfree(kid_tab, cap_kid_tab); dfree(sort_mode, cap_sort_mode); dfree(sort_gbase, cap_sort_gbase);
    dfree(hist, cap_hist); dfree(sort_status, cap_status); dfree(tile_hist, cap_tile_hist); dfree(scalars, cap_scalars);
    dfree(scan_scratch, cap_scan); dfree(PS1, cap_ps1); dfree(PS2, cap_ps2); dfree(TB, cap_TB); dfree(chunk_sq, cap_chunk_sq);
    dfree(cut, cap_cut); dfree(cut_SL, cap_cut_SL); dfree(cut_QL, cap_cut_QL); dfree(cnt_sz, cap_cntsz); dfree(flags, cap_flags);
    dfree(leaf_lo, cap_leaf_lo); dfree(leaf_m, cap_leaf_m); dfree(leaf_moff, cap_leaf_moff);
    dfree(leaf_U, cap_leaf_U); dfree(leaf_census, cap_leaf_census); dfree(leaf_kid, cap_leaf_kid);
    dfree(leaf_ord, cap_leaf_ord); dfree(fix_acc, cap_fix); dfree(kern_T, cap_kern_T); dfree(kern_g, cap_kern_g);
    dfree(red_part, cap_red); dfree(out_clusters, cap_out_cl); dfree(out_row, cap_out_row);
    dfree(out_cluster, cap_out_cluster); dfree(out_weight, cap_out_weight);
    dfree(big_ent, cap_big_ent); dfree(big_part, cap_big_part); dfree(big_thr, cap_big_thr);
    dfree(peer_dst, cap_peer_dst);
    dfree(vr_P, cap_vr_P); dfree(vr_work, cap_vr_work); dfree(gi_buf, cap_gi_buf);
    dfree(dn_sel, cap_dn_sel); dfree(dn_meta, cap_dn_meta); dfree(dn_val, cap_dn_val);
    dfree(gi_tab, cap_gi_tab); dfree(gi_rec, cap_gi_rec); dfree(gi_all, cap_gi_all); dfree(gi_val, cap_gi_val);
    dfree(km_dpos, cap_km_dpos); dfree(km_arg, cap_km_arg); dfree(km_ngrp, cap_km_ngrp);
    dfree(km_dP, cap_km_dP); dfree(km_F, cap_km_F); dfree(km_meta, cap_km_meta); dfree(km_sub, cap_km_sub);
    dfree(part_cnt, cap_part_cnt); dfree(dist_cnt, cap_dist_cnt);
    for (int i = 0; i < 3; i++) { dfree(xfer_u32[i], cap_xfer_u32[i]); dfree(recv_u32[i], cap_recv_u32[i]); }
    dfree(xfer_f64, cap_xfer_f64); dfree(xfer_f64b, cap_xfer_f64b); dfree(red_part2, cap_red2);
    dfree(g_clusters, cap_g_clusters); dfree(g_row, cap_g_row); dfree(g_cluster, cap_g_cluster);
    dfree(g_weight, cap_g_weight);
    dfree(mb_first, cap_mb_first); dfree(mb_lo, cap_mb_lo); dfree(mb_gkid, cap_mb_gkid);
    dfree(mb_leaf_of, cap_mb_leaf_of); dfree(mb_n, cap_mb_n); dfree(mb_gm, cap_mb_gm);
    dfree(mb_acc, cap_mb_acc); dfree(mb_part, cap_mb_part); dfree(mb_rec, cap_mb_rec);
    mb_m = nullptr;
}

// z = Phi^-1(1 - q), q = (1-conf)/2: Acklam's rational initial guess for the
// lower tail, refined by Halley steps on erfc (host; the oracle uses AS241).
static double z_two_sided(double conf) {
    const double q = 0.5 * (1.0 - conf);   // lower-tail probability, accurate for conf near 1
    static const double a[] = {-3.969683028665376e+01, 2.209460984245205e+02, -2.759285104469687e+02,
                               1.383577518672690e+02, -3.066479806614716e+01, 2.506628277459239e+00};
    static const double b[] = {-5.447609879822406e+01, 1.615858368580409e+02, -1.556989798598866e+02,
                               6.680131188771972e+01, -1.328068155288572e+01};
    static const double c[] = {-7.784894002430293e-03, -3.223964580411365e-01, -2.400758277161838e+00,
                               -2.549732539343734e+00, 4.374664141464968e+00, 2.938163982698783e+00};
    static const double d[] = {7.784695709041462e-03, 3.224671290700398e-01, 2.445134137142996e+00,
                               3.754408661907416e+00};
    double x;
    if (q < 0.02425) {
        const double r = std::sqrt(-2.0 * std::log(q));
        x = (((((c[0] * r + c[1]) * r + c[2]) * r + c[3]) * r + c[4]) * r + c[5]) /
            ((((d[0] * r + d[1]) * r + d[2]) * r + d[3]) * r + 1.0);
    } else {
        const double u = q - 0.5, r = u * u;
        x = (((((a[0] * r + a[1]) * r + a[2]) * r + a[3]) * r + a[4]) * r + a[5]) * u /
            (((((b[0] * r + b[1]) * r + b[2]) * r + b[3]) * r + b[4]) * r + 1.0);
    }
    for (int it = 0; it < 2; it++) {   // Halley on F(x) = Phi(x) - q, x < 0
        const double e = 0.5 * std::erfc(-x / std::sqrt(2.0)) - q;
        const double u = e * std::sqrt(2.0 * M_PI) * std::exp(0.5 * x * x);
        x = x - u / (1.0 + 0.5 * x * u);
    }
    return -x;
}

static int validate(const stem_trace *tr, double eps, double conf, const stem_opts &o) {
    if (!tr) return STEM_E_INVAL;
    if (!(eps > 0.0 && eps < 1.0)) return STEM_E_INVAL;
    if (!(o.z > 0.0) && !(conf > 0.0 && conf < 1.0)) return STEM_E_INVAL;
    if (o.z < 0.0 || std::isnan(o.z) || std::isinf(o.z)) return STEM_E_INVAL;
    if (o.scope < 0 || o.scope > 2) return STEM_E_INVAL;
    if (o.split < 0 || o.split > 3) return STEM_E_INVAL;
    if (o.split == 3 && (o.kmeans_k < 2 || o.kmeans_k > 8)) return STEM_E_INVAL;
    if (o.metric_bounds < 0 || o.metric_bounds > 1) return STEM_E_INVAL;
    if (tr->n == 0 || !tr->kernel_id || !tr->exec_ns) return STEM_E_INVAL;
    if (tr->n_metrics > 64 || (tr->n_metrics > 0 && !tr->metrics)) return STEM_E_INVAL;
    if (tr->n >= (1ull << 32)) return STEM_E_RANGE;
    if (tr->n_kernels == 0 || tr->n_kernels > (1u << 24)) return STEM_E_RANGE;
    return STEM_OK;
}

static int run_plan(Ctx &c, const stem_trace *tr, double eps, double conf, const stem_opts &o) {
    c.have_plan = false;
    c.launches = 0;
    c.stats = stem_stats{};
    c.timing.reset();
    CKS(validate(tr, eps, conf, o));
    CK(cudaSetDevice(c.device));
    if (tr->device >= 0 && tr->device != c.device) return STEM_E_INVAL;
    c.stream = (cudaStream_t)o.stream;
    const uint64_t n = tr->n;
    const uint32_t K = tr->n_kernels, nm = tr->n_metrics;
    double z = o.z;
    if (!(z > 0.0)) {
        z = z_two_sided(conf);
        if (!(z > 0.0) || std::isinf(z)) return STEM_E_INVAL;
    }
    const double q = z / eps;
    const double k2 = q * q;
    CKS(c.ensure_all(n, K, nm));
    const uint32_t *kid = tr->kernel_id, *t = tr->exec_ns;
    const double *met = tr->metrics;
    const uint32_t *h_kid = nullptr, *h_t = nullptr;
    if (tr->device < 0) {   // host trace: copied in by sort_trace, in chunks overlapped with its pre-pass
        CKS(c.ensure(c.in_kid, c.cap_in_kid, sizeof(uint32_t) * n));
        CKS(c.ensure(c.in_t, c.cap_in_t, sizeof(uint32_t) * n));
        h_kid = kid;
        h_t = t;
        kid = c.in_kid;
        t = c.in_t;
        if (nm) {
            CKS(c.ensure(c.in_met, c.cap_in_met, sizeof(double) * n * nm));
            CK(cudaMemcpyAsync(c.in_met, met, sizeof(double) * n * nm, cudaMemcpyHostToDevice, c.stream));
            met = c.in_met;
        }
    }
    CKS(sort_trace(c, kid, t, nullptr, n, K, !o.census_cap, h_kid, h_t));   // a1
    CKS(prefix_moments(c, n));                        // a2
    if (o.root && o.split == 3) {
        CKS(root_levels_kmeans(c, n, K, eps, z, k2, o.clamp_in_split ? 1 : 0, (uint32_t)o.kmeans_k));   // a3, a4
    } else if (o.root) {
        CKS(root_levels(c, n, K, eps, z, k2, o.clamp_in_split ? 1 : 0, o.split, o.seed));   // a3, a4
    } else {
        CKS(stem_only_leaves(c, n, K));
    }
    CKS(leaves_and_plan(c, n, K, met, nm, eps, z, k2, o, kid, t, n));   // a5 - a8
    c.n = n;
    c.K = K;
    c.n_metrics = nm;
    c.eps = eps;
    c.z = z;
    c.stats.kernel_launches = c.launches;
    c.stats.owned_rows = n;
    c.stats.world = 1;
    if (c.timing.on) {
        CK(cudaStreamSynchronize(c.stream));
        c.timing.finish();
    }
    c.have_plan = true;
    return STEM_OK;
}

// ---------------------------------------------------------------- host plans
// A plan is one header + one host block holding every array.  The block is
// page-locked (cudaMallocHost) so the plan's device-to-host copies run at full
// PCIe / C2C speed; freed blocks are kept in a small process-wide pool and
// reused by later plans, since pinning memory costs far more than copying it.
struct PlanBlock {
    stem_plan pub;     // first member: stem_plan_free casts back
    void *mem;
    size_t bytes;
    bool pinned;
};

struct PinnedPool {
    std::mutex m;
    std::vector<std::pair<void *, size_t>> free_blocks;   // (block, bytes)
    static constexpr size_t kKeep = 4;
};

static PinnedPool &pinned_pool() {
    static PinnedPool *p = new PinnedPool();   // never destroyed: blocks may outlive static teardown
    return *p;
}

static void *pool_acquire(size_t bytes, size_t &got, bool &pinned) {
    {
        PinnedPool &pp = pinned_pool();
        std::lock_guard<std::mutex> g(pp.m);
        int bi = -1;
        for (size_t i = 0; i < pp.free_blocks.size(); i++) {
            const size_t b = pp.free_blocks[i].second;
            if (b >= bytes && b <= 4 * bytes + (1u << 20) && (bi < 0 || b < pp.free_blocks[bi].second)) bi = (int)i;
        }
        if (bi >= 0) {
            void *m = pp.free_blocks[bi].first;
            got = pp.free_blocks[bi].second;
            pp.free_blocks.erase(pp.free_blocks.begin() + bi);
            pinned = true;
            return m;
        }
    }
    const size_t want = bytes + bytes / 8 + 4096;   // headroom: the next plan of the same trace reuses it
    void *m = nullptr;
    if (cudaMallocHost(&m, want) == cudaSuccess) {
        got = want;
        pinned = true;
        return m;
    }
    cudaGetLastError();
    pinned = false;
    got = bytes;
    return malloc(bytes);
}

static void pool_release(void *m, size_t bytes, bool pinned) {
    if (!m) return;
    if (!pinned) {
        free(m);
        return;
    }
    PinnedPool &pp = pinned_pool();
    std::lock_guard<std::mutex> g(pp.m);
    if (pp.free_blocks.size() < PinnedPool::kKeep) {
        pp.free_blocks.emplace_back(m, bytes);
        return;
    }
    cudaFreeHost(m);
}

// the plan block's layout for L clusters, S samples, nm metrics
struct PlanLayout {
    size_t o_cl, o_row, o_scl, o_w, o_est, o_tru, o_bnd, total;
    PlanLayout(uint64_t L, uint64_t S, uint64_t nm) {
        auto al = [](size_t x) { return (x + 63) & ~(size_t)63; };
        o_cl = 0;
        o_row = o_cl + al(sizeof(stem_cluster) * L);
        o_scl = o_row + al(sizeof(uint32_t) * S);
        o_w = o_scl + al(sizeof(uint32_t) * S);
        o_est = o_w + al(sizeof(double) * S);
        o_tru = o_est + al(sizeof(double) * (nm ? nm : 1));
        o_bnd = o_tru + al(sizeof(double) * nm);
        total = o_bnd + al(sizeof(double) * nm);
    }
};

static PlanBlock *plan_block_new(uint64_t L, uint64_t S, uint32_t nm) {
    PlanBlock *pb = (PlanBlock *)calloc(1, sizeof(PlanBlock));
    if (!pb) return nullptr;
    stem_plan *p = &pb->pub;
    const PlanLayout ly(L, S, nm);
    size_t got = 0;
    bool pinned = false;
    char *mem = (char *)pool_acquire(ly.total, got, pinned);
    if (!mem) {
        free(pb);
        return nullptr;
    }
    pb->mem = mem;
    pb->bytes = got;
    pb->pinned = pinned;
    p->n_clusters = L;
    p->n_samples = S;
    p->clusters = (stem_cluster *)(mem + ly.o_cl);
    p->sample_row = (uint32_t *)(mem + ly.o_row);
    p->sample_cluster = (uint32_t *)(mem + ly.o_scl);
    p->sample_weight = (double *)(mem + ly.o_w);
    p->n_metrics = nm;
    p->est_metric = (double *)(mem + ly.o_est);
    p->true_metric = (double *)(mem + ly.o_tru);
    p->bound_metric = (double *)(mem + ly.o_bnd);
    return pb;
}

int plan_block_begin(Ctx &c, uint64_t L, uint64_t S, uint32_t nm, stem_cluster **clusters_dst, uint32_t **row_dst,
                     uint32_t **cl_dst, double **w_dst) {
    plan_block_abort(c);
    PlanBlock *pb = plan_block_new(L, S, nm);
    if (!pb) return STEM_E_NOMEM;
    c.early_plan = pb;
    *clusters_dst = pb->pub.clusters;
    *row_dst = pb->pub.sample_row;
    *cl_dst = pb->pub.sample_cluster;
    *w_dst = pb->pub.sample_weight;
    return STEM_OK;
}

void plan_block_abort(Ctx &c) {
    if (!c.early_plan) return;
    if (c.dstream) cudaStreamSynchronize(c.dstream);   // no copy may land in a released block
    cudaStreamSynchronize(c.stream);
    stem_plan_free(&((PlanBlock *)c.early_plan)->pub);
    c.early_plan = nullptr;
}

static int to_host(Ctx &c, stem_plan **out) {
    const uint64_t L = c.n_leaves, S = c.n_samples;
    PlanBlock *pb = (PlanBlock *)c.early_plan;
    c.early_plan = nullptr;
    cudaError_t e = cudaSuccess;
    if (pb) {   // every copy already queued (leaves_and_plan): wait for them
        if (c.dstream) e = cudaStreamSynchronize(c.dstream);
        if (e == cudaSuccess) e = cudaStreamSynchronize(c.stream);
    } else {
        pb = plan_block_new(L, S, c.n_metrics);
        if (!pb) return STEM_E_NOMEM;
        stem_plan *p = &pb->pub;
        cudaStream_t st = c.stream;
        if (L) e = cudaMemcpyAsync(p->clusters, c.out_clusters, sizeof(stem_cluster) * L, cudaMemcpyDeviceToHost, st);
        if (S && e == cudaSuccess)
            e = cudaMemcpyAsync(p->sample_row, c.out_row, sizeof(uint32_t) * S, cudaMemcpyDeviceToHost, st);
        if (S && e == cudaSuccess)
            e = cudaMemcpyAsync(p->sample_cluster, c.out_cluster, sizeof(uint32_t) * S, cudaMemcpyDeviceToHost, st);
        if (S && e == cudaSuccess)
            e = cudaMemcpyAsync(p->sample_weight, c.out_weight, sizeof(double) * S, cudaMemcpyDeviceToHost, st);
        if (e == cudaSuccess) e = cudaStreamSynchronize(st);
    }
    stem_plan *p = &pb->pub;
    if (e != cudaSuccess) {
        last_cuda_error() = e;
        stem_plan_free(p);
        return STEM_E_CUDA;
    }
    if (!c.have_mbounds) {
        p->true_metric = nullptr;
        p->bound_metric = nullptr;
    }
    p->est_total_ns = c.est_total;
    p->true_total_ns = c.T;
    p->bound = c.bound;
    p->eps = c.eps;
    p->z = c.z;
    memcpy(p->est_metric, c.host_est_metric, sizeof(double) * c.n_metrics);
    if (c.have_mbounds) {
        memcpy(p->true_metric, c.host_true_metric, sizeof(double) * c.n_metrics);
        memcpy(p->bound_metric, c.host_bound_metric, sizeof(double) * c.n_metrics);
    }
    *out = p;
    return STEM_OK;
}

}  // namespace sr

struct stem_ctx {
    sr::Ctx c;
};

sr::Comm *stem_comm_impl(stem_comm *c);   // dist.cu

extern "C" {

int stem_default_opts(stem_opts *o) {
    if (!o) return STEM_E_INVAL;
    *o = stem_opts{};
    o->seed = 0;
    o->z = 0.0;
    o->scope = 0;
    o->root = 1;
    o->clamp_in_split = 1;
    o->census_cap = 0;
    o->split = 0;
    o->metric_bounds = 0;
    o->kmeans_k = 3;
    o->stream = nullptr;
    return STEM_OK;
}

int stem_ctx_create(int device, stem_ctx **out) {
    if (!out) return STEM_E_INVAL;
    *out = nullptr;
    int ndev = 0;
    cudaError_t e = cudaGetDeviceCount(&ndev);
    if (e != cudaSuccess) { sr::last_cuda_error() = e; return STEM_E_CUDA; }
    if (device < 0 || device >= ndev) return STEM_E_INVAL;
    stem_ctx *x = new (std::nothrow) stem_ctx();
    if (!x) return STEM_E_NOMEM;
    x->c.device = device;
    e = cudaSetDevice(device);
    if (e == cudaSuccess) e = cudaDeviceGetAttribute(&x->c.sms, cudaDevAttrMultiProcessorCount, device);
    if (e != cudaSuccess) {
        sr::last_cuda_error() = e;
        delete x;
        return STEM_E_CUDA;
    }
    *out = x;
    return STEM_OK;
}

void stem_ctx_destroy(stem_ctx *ctx) {
    if (!ctx) return;
    cudaSetDevice(ctx->c.device);
    ctx->c.release();
    delete ctx;
}

int stem_root_plan_ctx(stem_ctx *ctx, const stem_trace *trace, double eps, double conf, const stem_opts *opts,
                       stem_plan **out) {
    if (out) *out = nullptr;
    if (!ctx) return STEM_E_INVAL;
    stem_opts o;
    if (opts) o = *opts; else stem_default_opts(&o);
    ctx->c.want_host = out != nullptr;
    int s = sr::run_plan(ctx->c, trace, eps, conf, o);
    ctx->c.want_host = false;
    if (s != STEM_OK) {
        sr::plan_block_abort(ctx->c);
        ctx->c.have_plan = false;
        return s;
    }
    if (out) return sr::to_host(ctx->c, out);
    sr::plan_block_abort(ctx->c);
    return STEM_OK;
}

int stem_root_plan_dist(stem_ctx *ctx, stem_comm *comm, const stem_trace *local_shard, uint64_t global_row_base,
                        double eps, double conf, const stem_opts *opts, stem_plan **out) {
    if (out) *out = nullptr;
    sr::Comm *cm = stem_comm_impl(comm);
    if (!ctx || !cm) return STEM_E_INVAL;   // no communicator: nothing to agree with
    stem_opts o;
    if (opts) o = *opts; else stem_default_opts(&o);
    sr::Ctx &c = ctx->c;
    c.have_plan = false;
    c.launches = 0;
    c.stats = stem_stats{};
    c.timing.reset();
    static const stem_trace empty{};
    const stem_trace *tr = local_shard ? local_shard : &empty;
    // argument checks are rank-local (a shard may be empty or bad on one rank
    // only): the status is agreed across ranks inside run_plan_dist, so every
    // rank returns the same error instead of leaving its peers in a collective
    int local = STEM_OK;
    if (!local_shard || !(eps > 0.0 && eps < 1.0) || (!(o.z > 0.0) && !(conf > 0.0 && conf < 1.0)) || o.z < 0.0 ||
        std::isnan(o.z) || std::isinf(o.z) || o.scope < 0 || o.scope > 2 || o.split < 0 || o.split > 3 ||
        (o.split == 3 && (o.kmeans_k < 2 || o.kmeans_k > 8)) ||
        o.metric_bounds < 0 || o.metric_bounds > 1 || tr->n_metrics > 64 ||
        (tr->n && (!tr->kernel_id || !tr->exec_ns)) || (tr->n && tr->n_metrics && !tr->metrics))
        local = STEM_E_INVAL;
    else if (tr->n >= (1ull << 32) || tr->n_kernels == 0 || tr->n_kernels > (1u << 24))
        local = STEM_E_RANGE;
    else if (tr->device >= 0 && tr->device != c.device)
        local = STEM_E_INVAL;
    if (cudaSetDevice(c.device) != cudaSuccess) local = STEM_E_CUDA;
    c.stream = (cudaStream_t)o.stream;
    double z = o.z;
    if (local == STEM_OK && !(z > 0.0)) z = sr::z_two_sided(conf);
    c.z = z;
    c.eps = eps;
    c.comm = cm;
    int s = sr::run_plan_dist(c, *cm, tr, global_row_base, eps, conf, o, local);
    c.comm = nullptr;
    c.kid_base = 0;
    if (s != STEM_OK) return s;
    c.n = tr->n;
    c.n_metrics = tr->n_metrics;
    c.stats.kernel_launches = c.launches;
    if (c.timing.on) {
        if (cudaStreamSynchronize(c.stream) != cudaSuccess) return STEM_E_CUDA;
        c.timing.finish();
    }
    c.have_plan = true;
    if (out && sr::comm_rank(cm) == 0) return sr::to_host(c, out);
    return STEM_OK;
}

int stem_root_plan(const stem_trace *trace, double eps, double conf, const stem_opts *opts, stem_plan **out) {
    if (out) *out = nullptr;
    if (!trace || !out) return STEM_E_INVAL;
    stem_ctx *ctx = nullptr;
    int s = stem_ctx_create(trace->device >= 0 ? trace->device : 0, &ctx);
    if (s != STEM_OK) return s;
    s = stem_root_plan_ctx(ctx, trace, eps, conf, opts, out);
    stem_ctx_destroy(ctx);
    return s;
}

int stem_ctx_device_plan(const stem_ctx *ctx, stem_device_plan *v) {
    if (!ctx || !v) return STEM_E_INVAL;
    if (!ctx->c.have_plan) return STEM_E_STATE;
    const sr::Ctx &c = ctx->c;
    v->n_clusters = c.n_leaves;
    v->n_samples = c.n_samples;
    v->clusters = c.out_clusters;
    v->sample_row = c.out_row;
    v->sample_cluster = c.out_cluster;
    v->sample_weight = c.out_weight;
    v->est_total_ns = c.est_total;
    v->bound = c.bound;
    v->eps = c.eps;
    v->z = c.z;
    v->true_total_ns = c.T;
    v->n_metrics = c.n_metrics;
    v->est_metric = c.host_est_metric;
    v->true_metric = c.have_mbounds ? c.host_true_metric : nullptr;
    v->bound_metric = c.have_mbounds ? c.host_bound_metric : nullptr;
    return STEM_OK;
}

int stem_ctx_stats(const stem_ctx *ctx, stem_stats *s) {
    if (!ctx || !s) return STEM_E_INVAL;
    *s = ctx->c.stats;
    return STEM_OK;
}

int stem_ctx_enable_timing(stem_ctx *ctx, int on) {
    if (!ctx) return STEM_E_INVAL;
    ctx->c.timing.on = on != 0;
    return STEM_OK;
}

int stem_ctx_stage_times(const stem_ctx *ctx, stem_stage_time *out, uint32_t cap, uint32_t *count) {
    if (!ctx || !count || (cap && !out)) return STEM_E_INVAL;
    const auto &agg = ctx->c.timing.agg;
    *count = (uint32_t)agg.size();
    for (uint32_t i = 0; i < cap && i < agg.size(); i++) {
        memset(&out[i], 0, sizeof(stem_stage_time));
        strncpy(out[i].name, agg[i].name, sizeof(out[i].name) - 1);
        out[i].ms = agg[i].ms;
        out[i].bytes = agg[i].bytes;
        out[i].launches = agg[i].launches;
        out[i].count = agg[i].count;
    }
    return STEM_OK;
}

void stem_plan_free(stem_plan *p) {
    if (!p) return;
    sr::PlanBlock *pb = reinterpret_cast<sr::PlanBlock *>(p);   // every plan is a PlanBlock (to_host)
    sr::pool_release(pb->mem, pb->bytes, pb->pinned);
    free(pb);
}

const char *stem_strerror(int status) {
    switch (status) {
        case STEM_OK: return "ok";
        case STEM_E_INVAL: return "invalid argument";
        case STEM_E_RANGE: return "value out of range (n, n_kernels or a kernel_id)";
        case STEM_E_NOMEM: return "out of memory";
        case STEM_E_CUDA: return "CUDA error";
        case STEM_E_NCCL: return "NCCL error";
        case STEM_E_LIMIT: return "sample count limit (2^32) exceeded";
        case STEM_E_STATE: return "no plan has been built on this context";
        default: return "unknown status";
    }
}

int stem_z_from_conf(double conf, double *z_out) {
    if (!z_out) return STEM_E_INVAL;
    *z_out = 0.0;
    if (!(conf > 0.0 && conf < 1.0)) return STEM_E_INVAL;
    *z_out = sr::z_two_sided(conf);
    return STEM_OK;
}

}  // extern "C"
