// Device-wide exclusive scan and stable bucket partition (our own kernels; no CUB).
#pragma once
#include "common.cuh"

namespace spg {

constexpr int kScanThreads = 256;
constexpr int kScanItems = 8;
constexpr int kScanTile = kScanThreads * kScanItems;  // 2048

// Pass 1: per-tile sums (striped, coalesced loads).
template <typename Tin>
__global__ void __launch_bounds__(kScanThreads) k_scan_tile_sums(const Tin *__restrict__ in, int64_t n,
                                                                 int64_t *__restrict__ tile_sums) {
    __shared__ int64_t sm[kScanThreads / 32 + 1];
    const int64_t base = (int64_t)blockIdx.x * kScanTile;
    int64_t s = 0;
#pragma unroll
    for (int j = 0; j < kScanItems; ++j) {
        int64_t idx = base + j * kScanThreads + threadIdx.x;
        if (idx < n) s += (int64_t)in[idx];
    }
    s = warp_sum(s);
    if (lane_id() == 0) sm[warp_id()] = s;
    __syncthreads();
    if (threadIdx.x == 0) {
        int64_t t = 0;
        for (int w = 0; w < kScanThreads / 32; ++w) t += sm[w];
        tile_sums[blockIdx.x] = t;
    }
}

// Pass 2: exclusive scan of the tile sums in place (one block, chunked with carry);
// tile_sums[ntiles] receives the grand total.
__global__ void __launch_bounds__(1024) k_scan_spine(int64_t *__restrict__ tile_sums, int64_t ntiles) {
    __shared__ int64_t sm[1024 / 32 + 1];
    int64_t carry = 0;
    for (int64_t base = 0; base < ntiles; base += 1024) {
        int64_t idx = base + threadIdx.x;
        int64_t v = idx < ntiles ? tile_sums[idx] : 0;
        int64_t tot;
        int64_t ex = block_excl_sum<1024>(v, sm, &tot);
        if (idx < ntiles) tile_sums[idx] = carry + ex;
        carry += tot;
    }
    if (threadIdx.x == 0) tile_sums[ntiles] = carry;
}

// Pass 3: out[i] = tile_offset + exclusive prefix within the tile; out[n] = total.
template <typename Tin>
__global__ void __launch_bounds__(kScanThreads) k_scan_apply(const Tin *__restrict__ in, int64_t n,
                                                             const int64_t *__restrict__ tile_off,
                                                             int64_t *__restrict__ out, int64_t ntiles) {
    __shared__ int64_t sm[kScanThreads / 32 + 1];
    const int64_t base = (int64_t)blockIdx.x * kScanTile;
    int64_t carry = tile_off[blockIdx.x];
#pragma unroll 1
    for (int j = 0; j < kScanItems; ++j) {
        int64_t idx = base + j * kScanThreads + threadIdx.x;
        int64_t v = idx < n ? (int64_t)in[idx] : 0;
        int64_t tot;
        int64_t ex = block_excl_sum<kScanThreads>(v, sm, &tot);
        if (idx < n) out[idx] = carry + ex;
        carry += tot;
    }
    if (blockIdx.x == ntiles - 1 && threadIdx.x == 0) out[n] = tile_off[ntiles];
}

// Stable partition by a per-item bucket id (< nb <= 255).  Tile = one 256-thread block.
constexpr int kPartThreads = 256;

__global__ void __launch_bounds__(kPartThreads) k_part_count(const uint8_t *__restrict__ bucket, int64_t n,
                                                             int nb, int32_t *__restrict__ counts,
                                                             int64_t ntiles) {
    __shared__ int c[256];
    for (int b = threadIdx.x; b < nb; b += kPartThreads) c[b] = 0;
    __syncthreads();
    int64_t idx = (int64_t)blockIdx.x * kPartThreads + threadIdx.x;
    if (idx < n) atomicAdd(&c[bucket[idx]], 1);
    __syncthreads();
    for (int b = threadIdx.x; b < nb; b += kPartThreads) counts[(int64_t)b * ntiles + blockIdx.x] = c[b];
}

// offs = exclusive scan of counts ([nb][ntiles] bucket-major): bucket b begins at offs[b*ntiles].
__global__ void __launch_bounds__(kPartThreads) k_part_scatter(const uint8_t *__restrict__ bucket, int64_t n,
                                                               int nb, const int64_t *__restrict__ offs,
                                                               int64_t ntiles, int32_t *__restrict__ out) {
    constexpr int NW = kPartThreads / 32;
    __shared__ int wc[NW][256];
    for (int t = threadIdx.x; t < NW * 256; t += kPartThreads) (&wc[0][0])[t] = 0;
    __syncthreads();
    int64_t idx = (int64_t)blockIdx.x * kPartThreads + threadIdx.x;
    bool valid = idx < n;
    int b = valid ? (int)bucket[idx] : 255;
    unsigned peers = __match_any_sync(0xffffffffu, b);
    int rank = __popc(peers & lanemask_lt());
    if (valid && rank == 0) wc[warp_id()][b] = __popc(peers);
    __syncthreads();
    if (valid) {
        int pre = 0;
        for (int w = 0; w < warp_id(); ++w) pre += wc[w][b];
        out[offs[(int64_t)b * ntiles + blockIdx.x] + pre + rank] = (int32_t)idx;
    }
}

}  // namespace spg
