// sb.cu -- sort-stage (a1) microbenchmark: the library's sort_trace alone, with
// its per-stage CUDA events, over a device-resident trace.  Built with the
// library sources by tools/sortbench/sortbench.py (compile-time variants via -D).
#include <cstdio>
#include <cstring>

#include "../../paper_conf_micro_chungnkk25_b200/csrc/internal.h"

struct stem_ctx {
    sr::Ctx c;
};

// stage times averaged over reps - warm; names_out: nst_max x 32 chars
extern "C" __attribute__((visibility("default"))) int sb_sort(const uint32_t *kid, const uint32_t *t, uint64_t n,
                                                              uint32_t K, int warm, int reps, double *ms_out,
                                                              char *names_out, int nst_max, uint32_t *t_copy,
                                                              uint32_t *row_copy, int *pack_bits) {
    stem_ctx *ctx = nullptr;
    int s = stem_ctx_create(0, &ctx);
    if (s) return s;
    sr::Ctx &c = ctx->c;
    s = c.ensure_all(n, K, 0);
    int nst = 0;
    for (int r = 0; r < warm + reps && s == STEM_OK; r++) {
        c.timing.on = true;
        c.timing.reset();
        s = sr::sort_trace(c, kid, t, nullptr, n, K, true);
        if (s) break;
        if (cudaStreamSynchronize(c.stream) != cudaSuccess) { s = STEM_E_CUDA; break; }
        c.timing.finish();
        if (r < warm) continue;
        for (auto &g : c.timing.agg) {
            int j = 0;
            while (j < nst && strcmp(names_out + 32 * j, g.name)) j++;
            if (j == nst) {
                if (nst == nst_max) continue;
                strncpy(names_out + 32 * j, g.name, 31);
                ms_out[j] = 0;
                nst++;
            }
            ms_out[j] += g.ms / reps;
        }
    }
    if (s == STEM_OK && t_copy) cudaMemcpy(t_copy, c.t_sorted, 4 * n, cudaMemcpyDeviceToDevice);
    if (s == STEM_OK && row_copy) cudaMemcpy(row_copy, c.row_sorted, 4 * n, cudaMemcpyDeviceToDevice);
    if (pack_bits) *pack_bits = c.pack_s;
    stem_ctx_destroy(ctx);
    return s == STEM_OK ? -1000 - nst : s;   // < -1000: ok, stage count encoded
}
