// Device-wide exclusive scan and stable bucket partition (our own kernels; no CUB).
#pragma once
#include "common.cuh"

namespace spg {

constexpr int kScanThreads = 256;
constexpr int kScanItems = 8;
constexpr int kScanTile = kScanThreads * kScanItems;  // 2048

// Single-pass exclusive scan (decoupled look-back): tiles claimed in order by a ticket, each
// publishes its sum, resolves its prefix from its predecessors and writes out[]; out[n] = total.
// status[] (ntiles words) and ticket must be zero.
template <typename Tin>
__global__ void __launch_bounds__(kScanThreads) k_scan_onepass(const Tin *__restrict__ in, int64_t n,
                                                               int64_t *__restrict__ out,
                                                               unsigned long long *__restrict__ status,
                                                               unsigned long long *__restrict__ ticket) {
    __shared__ int64_t sm[kScanThreads / 32 + 1];
    __shared__ int64_t s_tile, s_pre;
    if (threadIdx.x == 0) s_tile = (int64_t)atomicAdd(ticket, 1ull);
    __syncthreads();
    const int64_t tile = s_tile;
    const int64_t b0 = tile * kScanTile + (int64_t)threadIdx.x * kScanItems;
    int64_t v[kScanItems];
    int64_t local = 0;
#pragma unroll
    for (int j = 0; j < kScanItems; ++j) {
        v[j] = b0 + j < n ? (int64_t)in[b0 + j] : 0;
        local += v[j];
    }
    int64_t tot;
    const int64_t ex = block_excl_sum<kScanThreads>(local, sm, &tot);
    if (warp_id() == 0) {
        lb_publish(status, tile, tot);
        const int64_t pre = lb_resolve(status, tile, tot);
        if (lane_id() == 0) s_pre = pre;
    }
    __syncthreads();
    int64_t run = s_pre + ex;
#pragma unroll
    for (int j = 0; j < kScanItems; ++j) {
        if (b0 + j < n) out[b0 + j] = run;
        run += v[j];
    }
    if (threadIdx.x == 0 && (tile + 1) * kScanTile >= n) out[n] = s_pre + tot;
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
