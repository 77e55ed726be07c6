// Stage (4): merge of Ĉ into C -- per row, sort by column + segmented reduce.
//
// PAPER.md §IV-D L452-L477 L: "elements with the same indices are merged into unique elements.
// This merging process is highly memory intensive ... B-Limiting ... limiting the number of
// blocks allocated to an SM ... extra shared memory ... applied only to the large rows of ĉ_i*".
// BASELINE.json north_star: "a row-bucketed sort plus segmented reduce into CSR".
//
// Every bin sorts the row's (col, val) pairs by col and reduces equal-col segments in fp64,
// rounding once to fp32; the merged row is written back in place at the start of the row's
// Ĉ bucket and its length to ccount[i].  Bins (rows of one class run one kernel):
//   warp      L <= 32        one warp, register bitonic network (shuffles)
//   warpradix L <= 512       one warp, stable LSD radix sort in the warp's smem slice
//   ctaradix  L <= t_lim     one CTA, stable LSD radix sort in smem (warp-ordered ranking)
//   limited   L >  t_lim     B-Limited: persistent CTAs with a 128 KB smem column window each
//                            (1 resident block per SM): dense fp64 window = counting sort with
//                            the segment reduction fused into the bucket accumulation.
#pragma once
#include "analysis.cuh"

namespace spg {

constexpr int32_t kKeyPad = 0x7fffffff;

// ------------------------------------------------------------------------ warp bin ---
__global__ void __launch_bounds__(256) k_merge_warp(const int32_t *__restrict__ rows, int64_t nrows,
                                                    const int64_t *__restrict__ rowoff, int32_t *__restrict__ chat_col,
                                                    float *__restrict__ chat_val, int64_t *__restrict__ ccount) {
    const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    if (gw >= nrows) return;
    const int lane = lane_id();
    const int i = rows[gw];
    const int64_t s = rowoff[i];
    const int L = (int)(rowoff[i + 1] - s);
    int32_t key = lane < L ? chat_col[s + lane] : kKeyPad;
    double v = lane < L ? (double)chat_val[s + lane] : 0.0;
    // bitonic sort of 32 (key, v) pairs, ascending by key
#pragma unroll
    for (int k = 2; k <= 32; k <<= 1) {
#pragma unroll
        for (int j = k >> 1; j > 0; j >>= 1) {
            int32_t pk = __shfl_xor_sync(0xffffffffu, key, j);
            double pv = __shfl_xor_sync(0xffffffffu, v, j);
            bool up = (lane & k) == 0;
            bool lower = (lane & j) == 0;
            bool take = lower == up ? (pk < key) : (pk > key);
            if (take) { key = pk; v = pv; }
        }
    }
    const int32_t prev = __shfl_up_sync(0xffffffffu, key, 1);
    const int32_t next = __shfl_down_sync(0xffffffffu, key, 1);
    const bool valid = key != kKeyPad;
    const bool head = lane == 0 || prev != key;
    const unsigned heads = __ballot_sync(0xffffffffu, head);
    const int seg_start = 31 - __clz(heads & (lanemask_lt() | (1u << lane)));
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
        double o = __shfl_up_sync(0xffffffffu, v, d);
        if (lane - d >= seg_start) v += o;
    }
    const bool tail = valid && (lane == 31 || next != key);
    const unsigned tails = __ballot_sync(0xffffffffu, tail);
    if (tail) {
        const int pos = __popc(tails & lanemask_lt());
        chat_col[s + pos] = key;
        chat_val[s + pos] = (float)v;
    }
    if (lane == 0) ccount[i] = __popc(tails);
}

// ------------------------------------------------------------- radix sort helpers ---
// Stable LSD radix pass over a[0..L) -> b, 8-bit digit of (key - kmin) >> shift, executed by
// a group of NW warps; warp w owns the contiguous chunk [w*C, (w+1)*C) and ranks equal
// digits inside a 32-element step with __match_any_sync (lane order = element order).
// cnt[w*256 + d]: per-warp digit counters.  Requires the caller to sync the group around it.
template <int NW>
struct RadixGroup {
    __device__ static void sync() {
        if constexpr (NW == 1) __syncwarp(); else __syncthreads();
    }
};

template <int NW>
__device__ __forceinline__ void radix_pass(const int32_t *ka, const float *va, int32_t *kb, float *vb, int L,
                                           int32_t kmin, int shift, int *cnt, int64_t *scan_sm, int gtid,
                                           int gwarp) {
    const int lane = lane_id();
    const int C = (L + NW - 1) / NW;
    const int c0 = min(L, gwarp * C), c1 = min(L, c0 + C);
    for (int t = gtid; t < NW * 256; t += NW * 32) cnt[t] = 0;
    RadixGroup<NW>::sync();
    for (int p = c0 + lane; p < c1; p += 32) {
        int d = ((ka[p] - kmin) >> shift) & 255;
        atomicAdd(&cnt[gwarp * 256 + d], 1);
    }
    RadixGroup<NW>::sync();
    if constexpr (NW == 1) {
        // warp scan over 256 digits: lane owns digits [8*lane, 8*lane+8)
        int loc[8];
        int sum = 0;
#pragma unroll
        for (int q = 0; q < 8; ++q) { loc[q] = cnt[lane * 8 + q]; sum += loc[q]; }
        int ex = warp_incl_sum(sum) - sum;
#pragma unroll
        for (int q = 0; q < 8; ++q) { cnt[lane * 8 + q] = ex; ex += loc[q]; }
    } else {
        // thread d (< 256) owns digit d across the NW warps
        int d = gtid;
        int tot = 0;
        if (d < 256)
            for (int w = 0; w < NW; ++w) tot += cnt[w * 256 + d];
        int64_t total;
        int64_t ex = block_excl_sum<NW * 32, int64_t>((int64_t)tot, scan_sm, &total);
        if (d < 256) {
            int run = (int)ex;
            for (int w = 0; w < NW; ++w) {
                int c = cnt[w * 256 + d];
                cnt[w * 256 + d] = run;
                run += c;
            }
        }
    }
    RadixGroup<NW>::sync();
    for (int p0 = c0; p0 < c1; p0 += 32) {
        const int p = p0 + lane;
        const bool ok = p < c1;
        int32_t k = ok ? ka[p] : 0;
        float v = ok ? va[p] : 0.f;
        int d = ok ? (((k - kmin) >> shift) & 255) : 256 + lane;
        unsigned peers = __match_any_sync(0xffffffffu, d);
        int rank = __popc(peers & lanemask_lt());
        int pos = ok ? cnt[gwarp * 256 + d] + rank : 0;
        __syncwarp();
        if (ok) {
            kb[pos] = k;
            vb[pos] = v;
            if (rank == 0) cnt[gwarp * 256 + d] += __popc(peers);
        }
        __syncwarp();
    }
    RadixGroup<NW>::sync();
}

// Segmented reduce of a sorted row kept in smem (k[0..L), v[0..L)) by a group of NW warps;
// writes the merged row to out_col/out_val[0..U) and returns U.  Each thread owns a contiguous
// run of ITEMS elements; a segment is summed in fp64 by the thread owning its head.
template <int NW>
__device__ __forceinline__ int segmented_reduce_out(const int32_t *k, const float *v, int L, int32_t kmin,
                                                    int32_t *__restrict__ out_col, float *__restrict__ out_val,
                                                    int64_t *scan_sm, int gtid) {
    constexpr int T = NW * 32;
    const int items = (L + T - 1) / T;
    const int p0 = min(L, gtid * items), p1 = min(L, p0 + items);
    int nh = 0;
    for (int p = p0; p < p1; ++p) nh += (p == 0 || k[p] != k[p - 1]);
    int total;
    int pos;
    if constexpr (NW == 1) {
        int inc = warp_incl_sum(nh);
        pos = inc - nh;
        total = __shfl_sync(0xffffffffu, inc, 31);
    } else {
        int64_t t64;
        pos = (int)block_excl_sum<T, int64_t>((int64_t)nh, scan_sm, &t64);
        total = (int)t64;
    }
    for (int p = p0; p < p1; ++p) {
        if (p == 0 || k[p] != k[p - 1]) {
            const int32_t key = k[p];
            double acc = (double)v[p];
            for (int q = p + 1; q < L && k[q] == key; ++q) acc += (double)v[q];
            out_col[pos] = key;
            out_val[pos] = (float)acc;
            ++pos;
        }
    }
    (void)kmin;
    return total;
}

// ------------------------------------------------------------------ warp radix bin ---
constexpr int kWarpRadixWarps = 8;
constexpr int kWarpRadixSmem = kWarpRadixWarps * (kWarpRadixMax * 16 + 256 * 4);

__global__ void __launch_bounds__(kWarpRadixWarps * 32) k_merge_warp_radix(
    const int32_t *__restrict__ rows, int64_t nrows, const int64_t *__restrict__ rowoff,
    int32_t *__restrict__ chat_col, float *__restrict__ chat_val, int64_t *__restrict__ ccount) {
    extern __shared__ __align__(16) unsigned char smem_raw[];
    const int w = warp_id(), lane = lane_id();
    unsigned char *my = smem_raw + w * (kWarpRadixMax * 16 + 256 * 4);
    int32_t *k0 = (int32_t *)my;
    float *v0 = (float *)(my + kWarpRadixMax * 4);
    int32_t *k1 = (int32_t *)(my + kWarpRadixMax * 8);
    float *v1 = (float *)(my + kWarpRadixMax * 12);
    int *cnt = (int *)(my + kWarpRadixMax * 16);
    const int64_t gw = (int64_t)blockIdx.x * kWarpRadixWarps + w;
    if (gw >= nrows) return;
    const int i = rows[gw];
    const int64_t s = rowoff[i];
    const int L = (int)(rowoff[i + 1] - s);
    int32_t mn = kKeyPad, mx = 0;
    for (int p = lane; p < L; p += 32) {
        int32_t c = chat_col[s + p];
        k0[p] = c;
        v0[p] = chat_val[s + p];
        mn = min(mn, c);
        mx = max(mx, c);
    }
    mn = warp_min(mn);
    mx = warp_max(mx);
    __syncwarp();
    const uint32_t span = (uint32_t)(mx - mn);
    const int bits = span ? 32 - __clz(span) : 0;
    for (int sh = 0; sh < bits; sh += 8) {
        radix_pass<1>(k0, v0, k1, v1, L, mn, sh, cnt, nullptr, lane, 0);
        int32_t *tk = k0; k0 = k1; k1 = tk;
        float *tv = v0; v0 = v1; v1 = tv;
    }
    const int U = segmented_reduce_out<1>(k0, v0, L, mn, chat_col + s, chat_val + s, nullptr, lane);
    if (lane == 0) ccount[i] = U;
}

// ------------------------------------------------------------------- CTA radix bin ---
constexpr int kCtaRadixThreads = 256;
constexpr int kCtaRadixWarps = kCtaRadixThreads / 32;

template <int CAP>
__global__ void __launch_bounds__(kCtaRadixThreads) k_merge_cta_radix(
    const int32_t *__restrict__ rows, int64_t nrows, const int64_t *__restrict__ rowoff,
    int32_t *__restrict__ chat_col, float *__restrict__ chat_val, int64_t *__restrict__ ccount) {
    extern __shared__ __align__(16) unsigned char smem_raw[];
    int32_t *k0 = (int32_t *)smem_raw;
    float *v0 = (float *)(smem_raw + CAP * 4);
    int32_t *k1 = (int32_t *)(smem_raw + CAP * 8);
    float *v1 = (float *)(smem_raw + CAP * 12);
    int *cnt = (int *)(smem_raw + CAP * 16);
    __shared__ int64_t scan_sm[kCtaRadixWarps + 1];
    __shared__ int32_t red_sm[kCtaRadixWarps];
    for (int64_t r = blockIdx.x; r < nrows; r += gridDim.x) {
        const int i = rows[r];
        const int64_t s = rowoff[i];
        const int L = (int)(rowoff[i + 1] - s);
        int32_t mn = kKeyPad, mx = 0;
        for (int p = threadIdx.x; p < L; p += kCtaRadixThreads) {
            int32_t c = chat_col[s + p];
            k0[p] = c;
            v0[p] = chat_val[s + p];
            mn = min(mn, c);
            mx = max(mx, c);
        }
        mn = block_reduce_min<kCtaRadixThreads>(mn, red_sm);
        mx = block_reduce_max<kCtaRadixThreads>(mx, red_sm);
        const uint32_t span = (uint32_t)(mx - mn);
        const int bits = span ? 32 - __clz(span) : 0;
        int32_t *ka = k0, *kb = k1;
        float *va = v0, *vb = v1;
        for (int sh = 0; sh < bits; sh += 8) {
            radix_pass<kCtaRadixWarps>(ka, va, kb, vb, L, mn, sh, cnt, scan_sm, threadIdx.x, warp_id());
            int32_t *tk = ka; ka = kb; kb = tk;
            float *tv = va; va = vb; vb = tv;
        }
        const int U = segmented_reduce_out<kCtaRadixWarps>(ka, va, L, mn, chat_col + s, chat_val + s, scan_sm,
                                                           threadIdx.x);
        if (threadIdx.x == 0) ccount[i] = U;
        __syncthreads();
    }
}

// ------------------------------------------------------------------- limited bin ---
// B-Limiting (L463-L477 L, Fig. 7): each block takes a 128 KB shared-memory column window so
// at most `limit_ctas_per_sm` (default 1) limited merge blocks are resident per SM; the grid is
// persistent (#SMs x limit) and claims rows longest-first from the limited list.
//
// Row i's Ĉ bucket is a set of runs (one per A entry (i,k)), each sorted by column (B's order).
// The block sweeps the row's column span in windows of S columns; per-run cursors advance
// monotonically, so every product is read once.  Inside a window the products are counted
// into their column bucket (fp64 accumulator + touched bit): a counting sort with the
// segment reduction fused into the bucket.  Emitting the set bits in order yields the
// window's merged, sorted output.  The merged row is staged in the block's private global
// scratch and copied back in place once the whole row has been read.
constexpr int kLimThreads = 512;
constexpr int kLimWindow = 16384;                       // columns per window (S)
constexpr int kLimSmem = kLimWindow * 8 + (kLimWindow / 32) * 4;

struct LimitedArgs {
    const int32_t *rows;          // limited rows, longest first
    int64_t nrows;
    const int64_t *rowoff;
    const int64_t *run_start;     // [nrows+1]
    const int64_t *run_base;
    const int32_t *run_len;
    int32_t *chat_col;
    float *chat_val;
    int64_t *ccount;
    int32_t *scratch_cursor;      // [grid][max_deg]
    int32_t *scratch_col;         // [grid][stage_cap]
    float *scratch_val;
    int64_t max_deg;
    int64_t stage_cap;
    unsigned long long *row_counter;
};

__device__ __forceinline__ void smem_add_f64(double *addr, double v) {
    unsigned long long *a = (unsigned long long *)addr;
    unsigned long long old = *a, assumed;
    do {
        assumed = old;
        old = atomicCAS(a, assumed, __double_as_longlong(__longlong_as_double(assumed) + v));
    } while (old != assumed);
}

__global__ void __launch_bounds__(kLimThreads, 1) k_merge_limited(LimitedArgs g) {
    extern __shared__ __align__(16) unsigned char smem_raw[];
    double *acc = (double *)smem_raw;
    uint32_t *bits = (uint32_t *)(smem_raw + kLimWindow * 8);
    __shared__ int64_t scan_sm[kLimThreads / 32 + 1];
    __shared__ int32_t red_sm[kLimThreads / 32];
    __shared__ int64_t row_sm;
    constexpr int NW = kLimThreads / 32;
    int32_t *cursor = g.scratch_cursor + (int64_t)blockIdx.x * g.max_deg;
    int32_t *st_col = g.scratch_col + (int64_t)blockIdx.x * g.stage_cap;
    float *st_val = g.scratch_val + (int64_t)blockIdx.x * g.stage_cap;
    for (int t = threadIdx.x; t < kLimWindow; t += kLimThreads) acc[t] = 0.0;
    for (int t = threadIdx.x; t < kLimWindow / 32; t += kLimThreads) bits[t] = 0u;
    const int lane = lane_id(), w = warp_id();
    while (true) {
        if (threadIdx.x == 0) row_sm = (int64_t)atomicAdd(g.row_counter, 1ull);
        __syncthreads();
        const int64_t r = row_sm;
        __syncthreads();
        if (r >= g.nrows) break;
        const int i = g.rows[r];
        const int64_t rs = g.run_start[r], R = g.run_start[r + 1] - rs;
        const int64_t *rbase = g.run_base + rs;
        const int32_t *rlen = g.run_len + rs;
        // column span of the row: first / last column of every run
        int32_t mn = kKeyPad, mx = 0;
        for (int64_t q = threadIdx.x; q < R; q += kLimThreads) {
            const int64_t b = rbase[q];
            mn = min(mn, g.chat_col[b]);
            mx = max(mx, g.chat_col[b + rlen[q] - 1]);
            cursor[q] = 0;
        }
        mn = block_reduce_min<kLimThreads>(mn, red_sm);
        mx = block_reduce_max<kLimThreads>(mx, red_sm);
        int64_t nout = 0;
        for (int64_t w0 = mn; w0 <= mx; w0 += kLimWindow) {
            const int32_t wend = (int32_t)min((int64_t)mx + 1, w0 + kLimWindow);
            // sweep: warp per run, 128 products per step (4 loads in flight per lane)
            for (int64_t q = w; q < R; q += NW) {
                const int64_t b = rbase[q];
                const int len = rlen[q];
                int cur = cursor[q];
                while (cur < len) {
                    int32_t c[4];
                    float v[4];
#pragma unroll
                    for (int u = 0; u < 4; ++u) {
                        const int p = cur + u * 32 + lane;
                        c[u] = p < len ? g.chat_col[b + p] : kKeyPad;
                        v[u] = p < len ? g.chat_val[b + p] : 0.f;
                    }
                    int taken = 0;
#pragma unroll
                    for (int u = 0; u < 4; ++u) {
                        const bool in = c[u] < wend;
                        if (in) {
                            const int x = c[u] - (int32_t)w0;
                            smem_add_f64(acc + x, (double)v[u]);
                            atomicOr(bits + (x >> 5), 1u << (x & 31));
                        }
                        taken += __popc(__ballot_sync(0xffffffffu, in));
                    }
                    cur += taken;
                    if (taken < 128) break;
                }
                if (lane == 0) cursor[q] = cur;
            }
            __syncthreads();
            // emit the window's touched columns in ascending order
            constexpr int WPT = (kLimWindow / 32) / kLimThreads;  // bit words per thread
            int cntw = 0;
            uint32_t word[WPT > 0 ? WPT : 1];
#pragma unroll
            for (int u = 0; u < WPT; ++u) {
                word[u] = bits[threadIdx.x * WPT + u];
                cntw += __popc(word[u]);
            }
            int64_t tot;
            int64_t pos = nout + block_excl_sum<kLimThreads, int64_t>((int64_t)cntw, scan_sm, &tot);
#pragma unroll
            for (int u = 0; u < WPT; ++u) {
                uint32_t m = word[u];
                while (m) {
                    const int bpos = __ffs(m) - 1;
                    m &= m - 1;
                    const int x = (threadIdx.x * WPT + u) * 32 + bpos;
                    st_col[pos] = (int32_t)w0 + x;
                    st_val[pos] = (float)acc[x];
                    acc[x] = 0.0;
                    ++pos;
                }
                bits[threadIdx.x * WPT + u] = 0u;
            }
            nout += tot;
            __syncthreads();
        }
        // copy the merged row back into the head of its Ĉ bucket
        const int64_t s = g.rowoff[i];
        for (int64_t p = threadIdx.x; p < nout; p += kLimThreads) {
            g.chat_col[s + p] = st_col[p];
            g.chat_val[s + p] = st_val[p];
        }
        if (threadIdx.x == 0) g.ccount[i] = nout;
        __syncthreads();
    }
}

// Single-run rows: already sorted and duplicate-free; merged length = bucket length.
__global__ void k_merge_pass(const int32_t *__restrict__ rows, int64_t nrows, const int64_t *__restrict__ rowoff,
                             int64_t *__restrict__ ccount) {
    for (int64_t q = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; q < nrows; q += (int64_t)gridDim.x * blockDim.x) {
        const int i = rows[q];
        ccount[i] = rowoff[i + 1] - rowoff[i];
    }
}

// ------------------------------------------------------------------ CSR compaction ---
// Output entry q of C belongs to row r with crowptr[r] <= q < crowptr[r+1]; it is read from
// Ĉ[rowoff[r] + q - crowptr[r]].  Tiles of 2048 outputs per block, rows found by binary search.
constexpr int kCompactThreads = 256;
constexpr int kCompactTile = 2048;

__global__ void __launch_bounds__(kCompactThreads) k_compact(const int64_t *__restrict__ crowptr, int64_t M,
                                                             const int64_t *__restrict__ rowoff,
                                                             const int32_t *__restrict__ chat_col,
                                                             const float *__restrict__ chat_val, int64_t nnz_c,
                                                             int32_t *__restrict__ out_col, float *__restrict__ out_val) {
    __shared__ int64_t lohi[2];
    const int64_t q0 = (int64_t)blockIdx.x * kCompactTile;
    const int64_t q1 = min(nnz_c, q0 + kCompactTile);
    if (threadIdx.x == 0) lohi[0] = upper_bound_idx(crowptr, 0, M, q0);
    if (threadIdx.x == 1) lohi[1] = upper_bound_idx(crowptr, 0, M, q1 - 1);
    __syncthreads();
    const int64_t lo = lohi[0], hi = lohi[1] + 1;
    for (int64_t q = q0 + threadIdx.x; q < q1; q += kCompactThreads) {
        const int64_t r = upper_bound_idx(crowptr, lo, hi, q);
        const int64_t src = rowoff[r] + (q - crowptr[r]);
        out_col[q] = chat_col[src];
        out_val[q] = chat_val[src];
    }
}

}  // namespace spg
