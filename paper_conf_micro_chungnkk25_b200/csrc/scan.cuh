// scan.cuh -- device-wide exclusive scan (reduce, scan of tile totals, apply).
// Input and output are functors so one primitive serves offsets, compactions
// and the exact prefix moments.  Three launches; tile = 256 threads x ITEMS.
#pragma once
#include "common.cuh"

namespace sr {

constexpr int kScanThreads = 256;
constexpr int kScanItems = 8;
constexpr uint64_t kScanTile = (uint64_t)kScanThreads * kScanItems;

template <class T, class In>
__global__ void __launch_bounds__(kScanThreads) scan_reduce_kernel(In in, uint64_t n, T *tile_tot) {
    __shared__ T sm[kScanThreads / 32 + 1];
    const uint64_t base = (uint64_t)blockIdx.x * kScanTile;
    T acc{};
#pragma unroll
    for (int j = 0; j < kScanItems; j++) {
        const uint64_t i = base + (uint64_t)j * kScanThreads + threadIdx.x;
        if (i < n) acc = acc + in(i);
    }
    T tot;
    block_excl_scan<T, kScanThreads>(acc, sm, &tot);
    if (threadIdx.x == 0) tile_tot[blockIdx.x] = tot;
}

// Single block: exclusive scan of tile totals in place; grand total to *total.
template <class T>
__global__ void __launch_bounds__(1024) scan_tiles_kernel(T *tile_tot, uint64_t ntiles, T *total) {
    __shared__ T sm[1024 / 32 + 1];
    T carry{};
    for (uint64_t b = 0; b < ntiles; b += 1024) {
        const uint64_t i = b + threadIdx.x;
        const T v = i < ntiles ? tile_tot[i] : T{};
        T tot;
        const T ex = block_excl_scan<T, 1024>(v, sm, &tot);
        if (i < ntiles) tile_tot[i] = carry + ex;
        carry = carry + tot;
    }
    if (threadIdx.x == 0) *total = carry;
}

// out(i, exclusive_prefix, value) for every i in [0, n), in any order.
template <class T, class In, class Out>
__global__ void __launch_bounds__(kScanThreads) scan_apply_kernel(In in, Out out, uint64_t n, const T *tile_tot) {
    __shared__ T sm[kScanThreads / 32 + 1];
    const uint64_t base = (uint64_t)blockIdx.x * kScanTile + (uint64_t)threadIdx.x * kScanItems;
    T v[kScanItems];
    T acc{};
#pragma unroll
    for (int j = 0; j < kScanItems; j++) {
        const uint64_t i = base + j;
        v[j] = i < n ? in(i) : T{};
        acc = acc + v[j];
    }
    T tot;
    T run = block_excl_scan<T, kScanThreads>(acc, sm, &tot);
    run = run + tile_tot[blockIdx.x];
#pragma unroll
    for (int j = 0; j < kScanItems; j++) {
        const uint64_t i = base + j;
        if (i < n) out(i, run, v[j]);
        run = run + v[j];
    }
}

// Scratch: ceil(n / kScanTile) T's for tile totals.  *total gets the sum.
inline uint64_t scan_tiles(uint64_t n) { return (n + kScanTile - 1) / kScanTile; }

template <class T, class In, class Out>
inline void exclusive_scan(In in, Out out, uint64_t n, T *tile_scratch, T *d_total, cudaStream_t st,
                           uint32_t *launches) {
    const uint64_t nt = scan_tiles(n);
    if (nt == 0) {
        cudaMemsetAsync(d_total, 0, sizeof(T), st);
        return;
    }
    scan_reduce_kernel<T, In><<<(unsigned)nt, kScanThreads, 0, st>>>(in, n, tile_scratch);
    scan_tiles_kernel<T><<<1, 1024, 0, st>>>(tile_scratch, nt, d_total);
    scan_apply_kernel<T, In, Out><<<(unsigned)nt, kScanThreads, 0, st>>>(in, out, n, tile_scratch);
    *launches += 3;
}

}  // namespace sr
