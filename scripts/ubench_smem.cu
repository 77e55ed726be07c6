// Shared-memory microbenchmarks on B200 (design input for the merge kernels; not product code).
// Each kernel runs ITERS warp-wide operations per warp on a 16K-int shared array; the report is
// SM-cycles per warp instruction (clock64 per CTA, max over CTAs) and lanes per SM-cycle.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o ubench_smem scripts/ubench_smem.cu
#include <cstdio>
#include <cuda_runtime.h>

constexpr int kWords = 16384;
constexpr int ITERS = 4096;

__device__ __forceinline__ unsigned hash32(unsigned x) {
    x ^= x >> 16; x *= 0x7feb352du; x ^= x >> 15; x *= 0x846ca68bu; x ^= x >> 16;
    return x;
}

template <int MODE>
__global__ void k_bench(unsigned *out, unsigned long long *cyc) {
    extern __shared__ unsigned s[];
    for (int q = threadIdx.x; q < kWords; q += blockDim.x) s[q] = 0;
    __syncthreads();
    unsigned acc = 0;
    unsigned h = hash32(threadIdx.x * 7919u + blockIdx.x);
    const long long t0 = clock64();
#pragma unroll 8
    for (int it = 0; it < ITERS; ++it) {
        h = h * 1664525u + 1013904223u;          // LCG: cheap distinct-ish addresses
        const unsigned idx = (h >> 8) & (kWords - 1);
        if constexpr (MODE == 0) acc += atomicAdd(&s[idx], 1u);            // ATOMS with return, spread
        else if constexpr (MODE == 1) atomicAdd(&s[idx], 1u);              // ATOMS no return, spread
        else if constexpr (MODE == 2) acc += s[idx];                       // LDS random
        else if constexpr (MODE == 3) s[idx] = h;                          // STS random
        else if constexpr (MODE == 4) acc += atomicAdd(&s[(threadIdx.x * 33 + it) & (kWords - 1)], 1u);  // conflict-free ATOMS
        else if constexpr (MODE == 5) { acc += s[(threadIdx.x * 33 + it) & (kWords - 1)]; }               // conflict-free LDS
        else if constexpr (MODE == 6) { if ((it & 15) == 0) __syncthreads(); acc += h; }                   // barrier every 16
        else if constexpr (MODE == 7) acc += atomicAdd(&s[idx & 1023], 1u);  // ATOMS, 1K words (more conflicts)
        else if constexpr (MODE == 8) { acc += __popc(__match_any_sync(0xffffffffu, idx >> 4)); }         // MATCH.ANY
    }
    const long long t1 = clock64();
    __syncthreads();
    out[blockIdx.x * blockDim.x + threadIdx.x] = acc + s[threadIdx.x];
    if ((threadIdx.x & 31) == 0) atomicMax(cyc, (unsigned long long)(t1 - t0));
}

template <int MODE>
void run(const char *name, int threads, int ctas_per_sm) {
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    const int grid = sms * ctas_per_sm;
    unsigned *out;
    unsigned long long *cyc;
    cudaMalloc(&out, (size_t)grid * threads * 4);
    cudaMalloc(&cyc, 8);
    const int smem = kWords * 4;
    cudaFuncSetAttribute(k_bench<MODE>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    k_bench<MODE><<<grid, threads, smem>>>(out, cyc);   // warm-up
    cudaMemset(cyc, 0, 8);
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    cudaEventRecord(a);
    k_bench<MODE><<<grid, threads, smem>>>(out, cyc);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms = 0;
    cudaEventElapsedTime(&ms, a, b);
    unsigned long long c = 0;
    cudaMemcpy(&c, cyc, 8, cudaMemcpyDeviceToHost);
    const double warp_instr_per_sm = (double)ctas_per_sm * (threads / 32) * ITERS;
    printf("%-28s threads=%4d ctas/sm=%d  cycles=%llu  SM-cyc/warp-op=%.2f  lanes/SM-cyc=%.2f  (%.3f ms) %s\n", name,
           threads, ctas_per_sm, c, c / warp_instr_per_sm, warp_instr_per_sm * 32 / c, ms,
           cudaGetErrorString(cudaGetLastError()));
    cudaFree(out);
    cudaFree(cyc);
}

int main() {
    for (int cps : {1, 2}) {
        run<0>("atoms_ret_spread", 1024, cps);
        run<1>("atoms_noret_spread", 1024, cps);
        run<2>("lds_random", 1024, cps);
        run<3>("sts_random", 1024, cps);
        run<4>("atoms_conflict_free", 1024, cps);
        run<5>("lds_conflict_free", 1024, cps);
        run<6>("bar_every16", 1024, cps);
        run<7>("atoms_ret_1k_words", 1024, cps);
        run<8>("match_any", 1024, cps);
    }
    run<0>("atoms_ret_spread", 256, 1);
    run<0>("atoms_ret_spread", 256, 4);
    run<2>("lds_random", 256, 4);
    return 0;
}
