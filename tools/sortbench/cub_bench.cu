// cub_bench.cu -- the library sort's yardstick: CUB's DeviceRadixSort (one-sweep
// on sm_100a) over n packed u64 keys of the same shape (38 key bits above 26 row
// bits), keys only and key + u32 value.  Times with CUDA events; prints ms.
#include <cstdio>
#include <cstdlib>
#include <cub/cub.cuh>

__global__ void fill(uint64_t *k, uint32_t *v, uint64_t n, uint64_t seed) {
    uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= n) return;
    uint64_t x = seed ^ (i * 0x9E3779B97F4A7C15ull);
    x ^= x >> 30; x *= 0xBF58476D1CE4E5B9ull; x ^= x >> 27; x *= 0x94D049BB133111EBull; x ^= x >> 31;
    k[i] = ((x >> 26) << 26) | (i & ((1ull << 26) - 1));
    v[i] = (uint32_t)i;
}

int main(int argc, char **argv) {
    const uint64_t n = argc > 1 ? strtoull(argv[1], 0, 10) : 1000000000ull;
    const int begin = argc > 2 ? atoi(argv[2]) : 26, end = argc > 3 ? atoi(argv[3]) : 64;
    uint64_t *k0, *k1; uint32_t *v0, *v1;
    cudaMalloc(&k0, 8 * n); cudaMalloc(&k1, 8 * n); cudaMalloc(&v0, 4 * n); cudaMalloc(&v1, 4 * n);
    fill<<<(unsigned)((n + 255) / 256), 256>>>(k0, v0, n, 1234);
    cub::DoubleBuffer<uint64_t> kb(k0, k1);
    cub::DoubleBuffer<uint32_t> vb(v0, v1);
    size_t t1 = 0, t2 = 0;
    cub::DeviceRadixSort::SortKeys(nullptr, t1, kb, (int64_t)n, begin, end);
    cub::DeviceRadixSort::SortPairs(nullptr, t2, kb, vb, (int64_t)n, begin, end);
    void *tmp; size_t tb = t1 > t2 ? t1 : t2; cudaMalloc(&tmp, tb);
    cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
    for (int mode = 0; mode < 2; mode++) {
        float best = 1e30f, sum = 0;
        for (int r = 0; r < 6; r++) {
            fill<<<(unsigned)((n + 255) / 256), 256>>>(kb.Current(), vb.Current(), n, 1234 + r);
            cudaEventRecord(a);
            if (mode == 0) cub::DeviceRadixSort::SortKeys(tmp, tb, kb, (int64_t)n, begin, end);
            else cub::DeviceRadixSort::SortPairs(tmp, tb, kb, vb, (int64_t)n, begin, end);
            cudaEventRecord(b); cudaEventSynchronize(b);
            float ms; cudaEventElapsedTime(&ms, a, b);
            if (r >= 1) { sum += ms; if (ms < best) best = ms; }
        }
        printf("cub %s n=%llu bits [%d,%d): mean %.3f ms, best %.3f ms (%s)\n", mode ? "SortPairs u64+u32" : "SortKeys u64",
               (unsigned long long)n, begin, end, sum / 5, best, cudaGetErrorString(cudaGetLastError()));
    }
    return 0;
}
