// Common device helpers for the B200 (sm_100a) spGEMM library.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

namespace spg {

constexpr int kWarp = 32;
constexpr int kNumSMs = 148;  // B200; the host queries the real count at plan time

__device__ __forceinline__ int lane_id() { return threadIdx.x & 31; }
__device__ __forceinline__ int warp_id() { return threadIdx.x >> 5; }

__device__ __forceinline__ unsigned lanemask_lt() {
    unsigned m;
    asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
    return m;
}

template <typename T>
__device__ __forceinline__ T warp_incl_sum(T v) {
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
        T o = __shfl_up_sync(0xffffffffu, v, d);
        if (lane_id() >= d) v += o;
    }
    return v;
}

template <typename T>
__device__ __forceinline__ T warp_sum(T v) {
#pragma unroll
    for (int d = 16; d > 0; d >>= 1) v += __shfl_xor_sync(0xffffffffu, v, d);
    return v;
}

template <typename T>
__device__ __forceinline__ T warp_min(T v) {
#pragma unroll
    for (int d = 16; d > 0; d >>= 1) v = min(v, __shfl_xor_sync(0xffffffffu, v, d));
    return v;
}

template <typename T>
__device__ __forceinline__ T warp_max(T v) {
#pragma unroll
    for (int d = 16; d > 0; d >>= 1) v = max(v, __shfl_xor_sync(0xffffffffu, v, d));
    return v;
}

// 32-bit integer reductions: one REDUX instruction instead of five shuffle rounds
template <>
__device__ __forceinline__ int warp_sum<int>(int v) { return __reduce_add_sync(0xffffffffu, v); }
template <>
__device__ __forceinline__ int warp_min<int>(int v) { return __reduce_min_sync(0xffffffffu, v); }
template <>
__device__ __forceinline__ int warp_max<int>(int v) { return __reduce_max_sync(0xffffffffu, v); }
template <>
__device__ __forceinline__ unsigned warp_sum<unsigned>(unsigned v) { return __reduce_add_sync(0xffffffffu, v); }
template <>
__device__ __forceinline__ unsigned warp_min<unsigned>(unsigned v) { return __reduce_min_sync(0xffffffffu, v); }
template <>
__device__ __forceinline__ unsigned warp_max<unsigned>(unsigned v) { return __reduce_max_sync(0xffffffffu, v); }

// Block-wide exclusive sum over THREADS threads; returns exclusive prefix, *total = sum.
// `smem` needs THREADS/32 + 1 slots.  Contains __syncthreads (all threads must call).
template <int THREADS, typename T>
__device__ __forceinline__ T block_excl_sum(T v, T *smem, T *total) {
    constexpr int NW = THREADS / 32;
    T inc = warp_incl_sum(v);
    if (lane_id() == 31) smem[warp_id()] = inc;
    __syncthreads();
    if (warp_id() == 0) {
        T w = lane_id() < NW ? smem[lane_id()] : T(0);
        T wi = warp_incl_sum(w);
        if (lane_id() < NW) smem[lane_id()] = wi - w;
        if (lane_id() == NW - 1) smem[NW] = wi;
    }
    __syncthreads();
    T r = smem[warp_id()] + inc - v;
    *total = smem[NW];
    __syncthreads();
    return r;
}

template <int THREADS, typename T>
__device__ __forceinline__ T block_reduce_min(T v, T *smem) {
    v = warp_min(v);
    if (lane_id() == 0) smem[warp_id()] = v;
    __syncthreads();
    T r = smem[0];
#pragma unroll
    for (int w = 1; w < THREADS / 32; ++w) r = min(r, smem[w]);
    __syncthreads();
    return r;
}

template <int THREADS, typename T>
__device__ __forceinline__ T block_reduce_max(T v, T *smem) {
    v = warp_max(v);
    if (lane_id() == 0) smem[warp_id()] = v;
    __syncthreads();
    T r = smem[0];
#pragma unroll
    for (int w = 1; w < THREADS / 32; ++w) r = max(r, smem[w]);
    __syncthreads();
    return r;
}

// Largest index i in [lo, hi) with ptr[i] <= x (ptr non-decreasing, ptr[lo] <= x).
__device__ __forceinline__ int64_t upper_bound_idx(const int64_t *__restrict__ ptr, int64_t lo, int64_t hi,
                                                   int64_t x) {
    // returns last i with ptr[i] <= x, searching i in [lo, hi)
    while (hi - lo > 1) {
        int64_t mid = (lo + hi) >> 1;
        if (__ldg(ptr + mid) <= x) lo = mid; else hi = mid;
    }
    return lo;
}

__device__ __forceinline__ int ilog2_floor(uint64_t x) { return 63 - __clzll((long long)x); }
__device__ __forceinline__ int ilog2_ceil(uint64_t x) { return x <= 1 ? 0 : 64 - __clzll((long long)(x - 1)); }

// ---- decoupled look-back (single-pass scans, the fused unit merge): a status word per tile,
// flag in the top 2 bits (1 aggregate, 2 inclusive prefix), value in the low 62.
constexpr unsigned long long kLbAgg = 1ull << 62, kLbPre = 2ull << 62, kLbMask = (1ull << 62) - 1;

__device__ __forceinline__ void st_release_u64(unsigned long long *p, unsigned long long v) {
    asm volatile("st.release.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ unsigned long long ld_acquire_u64(const unsigned long long *p) {
    unsigned long long v;
    asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}

// Decoupled look-back (one warp).  lb_publish: unit u's aggregate (unit 0: its inclusive
// prefix) as soon as its merged count is known; lb_resolve (later): sums predecessors'
// aggregates back to the nearest inclusive prefix, publishes u's inclusive prefix and returns the
// exclusive one.
__device__ __forceinline__ void lb_publish(unsigned long long *status, int64_t u, int64_t agg) {
    __threadfence();
    if (lane_id() == 0) st_release_u64(status + u, (u == 0 ? kLbPre : kLbAgg) | (unsigned long long)agg);
}
__device__ __forceinline__ int64_t lb_resolve(unsigned long long *status, int64_t u, int64_t agg) {
    if (u == 0) return 0;
    const int lane = lane_id();
    int64_t excl = 0;
    int64_t idx = u - 1 - lane;
    while (true) {
        unsigned long long s;
        while (true) {
            s = idx >= 0 ? ld_acquire_u64(status + idx) : kLbPre;
            if (!__any_sync(0xffffffffu, (s >> 62) == 0)) break;
            __nanosleep(64);   // (a spinning warp takes issue slots from the SM's other warps)
        }
        const unsigned pre = __ballot_sync(0xffffffffu, (s >> 62) == 2);
        int64_t v = (int64_t)(s & kLbMask);
        if (pre) {
            if (lane > __ffs(pre) - 1) v = 0;
            excl += warp_sum(v);
            break;
        }
        excl += warp_sum(v);
        idx -= 32;
    }
    if (lane == 0) st_release_u64(status + u, kLbPre | (unsigned long long)(excl + agg));
    return excl;
}

// ---- load balancing index (Eq. (3), L564-L577 R): LBI = (1/N) sum_i cycles(SM_i) /
// max cycles(SM), N = #SMs.  Opt-in recording (options.reserved[8] = 1): lbi[0] = the kernel's first
// CTA start, lbi[1 + smid] = the last CTA end on that SM (%globaltimer, ns); the host takes
// cycles(SM_i) = lbi[1 + i] - lbi[0].
constexpr int kLbiSlots = 1 + 256;
__device__ __forceinline__ unsigned long long gtimer_ns() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}
__device__ __forceinline__ unsigned sm_id() {
    unsigned s;
    asm volatile("mov.u32 %0, %%smid;" : "=r"(s));
    return s;
}
__device__ __forceinline__ void lbi_start(unsigned long long *lbi) {
    if (lbi && threadIdx.x == 0) atomicMin(lbi, gtimer_ns());
}
__device__ __forceinline__ void lbi_end(unsigned long long *lbi) {   // (uniform: lbi is a kernel argument)
    if (lbi) {
        __syncthreads();
        if (threadIdx.x == 0) atomicMax(lbi + 1 + (sm_id() & 255), gtimer_ns());
    }
}

}  // namespace spg
