// tracegen.cu -- CUDA twin of tracegen.generate_np (the specification).
// Input generator only: holds none of the STEM+ROOT arithmetic.  Per-row
// recipe is integer-only except metric columns, which use explicitly rounded
// fp64 mul/add (no FMA) so the bytes equal numpy's.
#include <cstdint>
#include <cuda_runtime.h>

namespace {

constexpr int kMaxPeak = 8;
constexpr int kTab = 4096;
constexpr int kFracBits = 20;
constexpr uint8_t kNoSitePeak = 0xFF;

__device__ __forceinline__ uint64_t splitmix(uint64_t x) {
    x += 0x9E3779B97F4A7C15ull;
    x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ull;
    x = (x ^ (x >> 27)) * 0x94D049BB133111EBull;
    return x ^ (x >> 31);
}

__device__ __forceinline__ uint64_t row_hash(uint64_t seed, uint64_t r, uint64_t stream) {
    return splitmix(seed ^ (r * 0xD1B54A32D192ED03ull) ^ (stream * 0x8CB92BA72F3D8DD7ull));
}

struct Params {
    uint64_t seed, row0, count;
    uint32_t n_sites, n_kernels, n_metrics;
    const uint32_t *site_kid;
    const uint8_t *site_peak;
    const uint32_t *pk_cum, *tail, *center;
    const uint16_t *ptab;
    const uint32_t *tables;
    const double *mA, *mB, *mS;
    const uint8_t *mclamp;
    uint32_t *kid_out, *t_out;
    double *met_out;
    uint64_t met_ld;
};

__global__ void __launch_bounds__(256) gen_kernel(Params p) {
    const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < p.count; i += stride) {
        const uint64_t r = p.row0 + i;
        const uint32_t site = (uint32_t)(r % p.n_sites);
        const uint32_t kid = __ldg(p.site_kid + site);
        const uint64_t h1 = row_hash(p.seed, r, 1);
        const uint32_t u_hi = (uint32_t)(h1 >> 32), u_lo = (uint32_t)h1;
        uint32_t peak = __ldg(p.site_peak + site);
        if (peak == kNoSitePeak) {
            peak = 0;
            while (peak < kMaxPeak - 1 && u_hi >= __ldg(p.pk_cum + kid * kMaxPeak + peak)) peak++;
        }
        if (u_lo < __ldg(p.tail + kid)) peak = kMaxPeak - 1;
        const uint32_t idx = kid * kMaxPeak + peak;
        const uint64_t h2 = row_hash(p.seed, r, 2);
        const uint32_t q = (uint32_t)(h2 >> 52);
        const uint64_t frac = (h2 >> 32) & ((1u << kFracBits) - 1);
        const uint64_t tb = (uint64_t)__ldg(p.ptab + idx) * (kTab + 1) + q;
        const uint64_t a = __ldg(p.tables + tb), b = __ldg(p.tables + tb + 1);
        const uint64_t v = a + (((b - a) * frac) >> kFracBits);
        uint64_t t = ((uint64_t)__ldg(p.center + idx) * v) >> kFracBits;
        if (t > 0xFFFFFFFFull) t = 0xFFFFFFFFull;
        p.kid_out[i] = kid;
        p.t_out[i] = (uint32_t)t;
        if (p.n_metrics) {
            const double tf = (double)(uint32_t)t;
            for (uint32_t c = 0; c < p.n_metrics; c++) {
                const double u = (double)(row_hash(p.seed, r, 3 + c) >> 11) * 0x1p-53;
                const uint64_t ck = (uint64_t)c * p.n_kernels + kid;
                const double x = __dmul_rn(__ldg(p.mA + ck), tf);
                const double y = __dmul_rn(__ldg(p.mS + ck), u);
                const double z = __dadd_rn(__ldg(p.mB + ck * kMaxPeak + peak), y);
                double val = __dadd_rn(x, z);
                if (p.mclamp[c]) val = fmin(fmax(val, 0.0), 1.0);
                p.met_out[(uint64_t)c * p.met_ld + i] = val;
            }
        }
    }
}

}  // namespace

extern "C" int tg_generate(uint64_t seed, uint64_t row0, uint64_t count, uint32_t n_sites,
                           const uint32_t *site_kid, const uint8_t *site_peak, const uint32_t *pk_cum,
                           const uint32_t *tail, const uint32_t *center, const uint16_t *ptab,
                           const uint32_t *tables, uint32_t n_kernels, uint32_t n_metrics,
                           const double *mA, const double *mB, const double *mS, const uint8_t *mclamp,
                           uint32_t *kid_out, uint32_t *t_out, double *met_out, uint64_t met_ld,
                           void *stream) {
    if (count == 0) return 0;
    Params p{seed, row0, count, n_sites, n_kernels, n_metrics, site_kid, site_peak, pk_cum, tail, center,
             ptab, tables, mA, mB, mS, mclamp, kid_out, t_out, met_out, met_ld};
    int dev = 0, sms = 148;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    uint64_t blocks = (count + 255) / 256;
    const uint64_t cap = (uint64_t)sms * 8;
    if (blocks > cap) blocks = cap;
    gen_kernel<<<(unsigned)blocks, 256, 0, (cudaStream_t)stream>>>(p);
    return cudaGetLastError() == cudaSuccess ? 0 : 1;
}
