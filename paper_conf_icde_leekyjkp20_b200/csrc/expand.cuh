// Stage (3): outer-product expansion into the row-bucketed intermediate matrix Ĉ.
//
// PAPER.md reconstructed Eq. (2) / Algorithm 1 (L150-L154, L325-L327 R): C = sum_k a_*k ⊗ b_k*;
// each product (i, j, a_ik*b_kj) is stored in Ĉ (L321-L323 L).  The row-wise offsets of
// stage (1) place every product of row i inside row i's bucket (L289-L291 R): the run of
// A entry e = (i, k) is Ĉ[base[e] .. base[e] + nnz(b_k*)), in B's (ascending) column order.
//
// Ĉ layout: SoA, row implicit: chat_col int32[nnz(Ĉ)], chat_val fp32[nnz(Ĉ)] (8 B/product).
// The kernels are store-bound: B values are held in registers, the A entries' (value, run
// base) pairs in shared memory, so the inner loop is stores only (no dependent loads).
#pragma once
#include "analysis.cuh"

namespace spg {

constexpr int kPieceThreads = 128;
constexpr int kPieceWarps = kPieceThreads / 32;
constexpr int kPieceAChunk = 256;   // A entries staged per round (= default split_ca_max)

// B-Split pieces and whole blocks (Normal pairs).  One CTA per piece.  The paper's block has
// nnz(b_k*) effective threads, each looping over the A column (L385-L386 R, L411-L415 L).
// Runs start 16-byte aligned (kRunAlign padding), so a lane owns 4 consecutive slots and
// writes them with one 16-byte store per array.
// Wide pieces (b_len >= 32): a warp holds a 128-slot chunk of the B sub-row in registers and
// streams it to every A entry of the piece (one int4 + one float4 store per lane and entry).
// Thin pieces (b_len < 32): micro-blocks of v lanes (v vectors cover the padded run) and 32/v
// A entries per warp step, so thin blocks do not idle lanes (block compaction, L406-L409 R).
// The slots after the run's last product (up to the padded length) get sentinel entries.
__device__ __forceinline__ void load_b4(const int32_t *__restrict__ bc, const float *__restrict__ bv, int j, int n,
                                        int4 &c4, float4 &v4) {
    c4.x = j + 0 < n ? __ldg(bc + j + 0) : 0x7fffffff;
    c4.y = j + 1 < n ? __ldg(bc + j + 1) : 0x7fffffff;
    c4.z = j + 2 < n ? __ldg(bc + j + 2) : 0x7fffffff;
    c4.w = j + 3 < n ? __ldg(bc + j + 3) : 0x7fffffff;
    v4.x = j + 0 < n ? __ldg(bv + j + 0) : 0.f;
    v4.y = j + 1 < n ? __ldg(bv + j + 1) : 0.f;
    v4.z = j + 2 < n ? __ldg(bv + j + 2) : 0.f;
    v4.w = j + 3 < n ? __ldg(bv + j + 3) : 0.f;
}

__device__ __forceinline__ void store_run4(int32_t *__restrict__ chat_col, float *__restrict__ chat_val, int64_t dst,
                                           const int4 &c4, const float4 &v4, float a) {
    *reinterpret_cast<int4 *>(chat_col + dst) = c4;
    *reinterpret_cast<float4 *>(chat_val + dst) = make_float4(a * v4.x, a * v4.y, a * v4.z, a * v4.w);
}

__global__ void __launch_bounds__(kPieceThreads) k_expand_pieces(
    const Piece *__restrict__ pieces, const float *__restrict__ a_val, const int64_t *__restrict__ b_rowptr,
    const int32_t *__restrict__ b_colidx, const float *__restrict__ b_val, const int64_t *__restrict__ base,
    int32_t *__restrict__ chat_col, float *__restrict__ chat_val) {
    __shared__ float s_a[kPieceAChunk];
    __shared__ int64_t s_dst[kPieceAChunk];
    const Piece pc = pieces[blockIdx.x];
    const int lane = lane_id(), w = warp_id();
    const int32_t *__restrict__ bc = b_colidx + pc.b_lo;
    const float *__restrict__ bv = b_val + pc.b_lo;
    // slots this piece writes: its B sub-row, plus the run's padding if it holds the last tile
    const int rb = (int)(__ldg(b_rowptr + pc.k + 1) - __ldg(b_rowptr + pc.k));
    const bool last = pc.b_off + pc.b_len == rb;
    const int nslots = last ? (int)pad_run(rb) - pc.b_off : pc.b_len;
    const bool vec = (pc.b_off % kRunAlign) == 0 && (nslots % kRunAlign) == 0;
    for (int a0 = 0; a0 < pc.a_len; a0 += kPieceAChunk) {
        const int na = min(kPieceAChunk, pc.a_len - a0);
        for (int t = threadIdx.x; t < na; t += kPieceThreads) {
            s_a[t] = __ldg(a_val + pc.a_lo + a0 + t);
            s_dst[t] = __ldg(base + pc.a_lo + a0 + t) + pc.b_off;
        }
        __syncthreads();
        if (!vec) {
            // B tiles not multiples of kRunAlign (a user split_b_tile): scalar stores
            for (int a = w; a < na; a += kPieceWarps)
                for (int j = lane; j < nslots; j += 32) {
                    const bool real = j < pc.b_len;
                    chat_col[s_dst[a] + j] = real ? __ldg(bc + j) : 0x7fffffff;
                    chat_val[s_dst[a] + j] = real ? s_a[a] * __ldg(bv + j) : 0.f;
                }
        } else if (pc.b_len >= 32) {
            const int nchunks = (nslots + 127) >> 7;
            const int slices = nchunks >= kPieceWarps ? 1 : kPieceWarps / nchunks;   // A slices per chunk
            for (int u = w; u < nchunks * slices; u += kPieceWarps) {
                const int j = ((u / slices) << 7) + 4 * lane;
                const int sl = u % slices;
                int4 c4;
                float4 v4;
                load_b4(bc, bv, j, pc.b_len, c4, v4);
                if (j < nslots)
                    for (int a = sl; a < na; a += slices) store_run4(chat_col, chat_val, s_dst[a] + j, c4, v4, s_a[a]);
            }
        } else {
            const int nvec = nslots >> 2;                       // 1..8 vectors per run
            const int shift = ilog2_ceil((uint64_t)nvec);       // micro-block of 2^shift lanes
            const int mb = lane >> shift;
            const int sub = lane & ((1 << shift) - 1);
            const int g = 32 >> shift;
            int4 c4;
            float4 v4;
            load_b4(bc, bv, 4 * sub, pc.b_len, c4, v4);
            if (sub < nvec)
                for (int a = w * g + mb; a < na; a += kPieceWarps * g)
                    store_run4(chat_col, chat_val, s_dst[a] + 4 * sub, c4, v4, s_a[a]);
        }
        __syncthreads();
    }
}

// B-Gathering (L369-L450): low performers with 2^(N-1) < nnz(b_k*) <= 2^N are packed into
// combined blocks ("gathering factor 32/2^n", L438-L441 L).  With 16-byte slots a lane covers
// 4 effective threads, so a micro-block is V = max(1, 2^N / 4) lanes and a warp packs 32 / V
// pairs; each micro-block keeps its B row in registers and loops over its A column, four A
// entries per step with their (value, base) loads issued together.
template <int N>
__global__ void __launch_bounds__(256) k_expand_gathered(
    const int32_t *__restrict__ list, int64_t count, const int64_t *__restrict__ a_colptr,
    const float *__restrict__ a_val, const int64_t *__restrict__ b_rowptr, const int32_t *__restrict__ b_colidx,
    const float *__restrict__ b_val, const int64_t *__restrict__ base, int32_t *__restrict__ chat_col,
    float *__restrict__ chat_val) {
    constexpr int V = (1 << N) >= 4 ? (1 << N) / 4 : 1;
    constexpr int SH = V == 1 ? 0 : (V == 2 ? 1 : (V == 4 ? 2 : 3));
    const int64_t slot = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> SH;
    const int sub = threadIdx.x & (V - 1);
    if (slot >= count) return;
    const int k = __ldg(list + slot);
    const int64_t a0 = __ldg(a_colptr + k), a1 = __ldg(a_colptr + k + 1);
    const int64_t b0 = __ldg(b_rowptr + k);
    const int rb = (int)(__ldg(b_rowptr + k + 1) - b0);
    if (4 * sub >= rb) return;
    int4 c4;
    float4 v4;
    load_b4(b_colidx + b0, b_val + b0, 4 * sub, rb, c4, v4);
    int64_t e = a0;
    for (; e + 4 <= a1; e += 4) {
        int64_t d[4];
        float av[4];
#pragma unroll
        for (int q = 0; q < 4; ++q) {
            d[q] = __ldg(base + e + q);
            av[q] = __ldg(a_val + e + q);
        }
#pragma unroll
        for (int q = 0; q < 4; ++q) store_run4(chat_col, chat_val, d[q] + 4 * sub, c4, v4, av[q]);
    }
    for (; e < a1; ++e) store_run4(chat_col, chat_val, __ldg(base + e) + 4 * sub, c4, v4, __ldg(a_val + e));
}

// B-Gathering, load-balanced: the items of gathering bin n are (pair, A entry) couples, laid out
// bin list order (pairs sorted by (n, c, k)) with item_off[q] = sum of nnz(a_*k) over earlier
// pairs of the gather lists.  One lane per item: it writes the pair's whole padded run (<= 8
// 16-byte vectors) for that A entry, so a warp combines 32 micro-blocks of up to 32 effective
// threads each and no lane loops over a long A column.
constexpr int kGatherTile = 512;
__global__ void __launch_bounds__(256) k_expand_gathered_items(
    const int32_t *__restrict__ list, const int64_t *__restrict__ item_off, int64_t q_lo, int64_t q_hi,
    const int64_t *__restrict__ a_colptr, const float *__restrict__ a_val, const int64_t *__restrict__ b_rowptr,
    const int32_t *__restrict__ b_colidx, const float *__restrict__ b_val, const int64_t *__restrict__ base,
    int32_t *__restrict__ chat_col, float *__restrict__ chat_val) {
    __shared__ int64_t s_off[kGatherTile + 1];
    __shared__ int64_t s_q0;
    __shared__ int s_n;
    const int64_t t_beg = item_off[q_lo], t_end = item_off[q_hi];
    const int64_t ntiles = (t_end - t_beg + kGatherTile - 1) / kGatherTile;
    for (int64_t tile = blockIdx.x; tile < ntiles; tile += gridDim.x) {
        const int64_t t0 = t_beg + tile * kGatherTile;
        if (threadIdx.x == 0) {
            int64_t lo = q_lo, hi = q_hi;     // pair of item t0: last q with item_off[q] <= t0
            while (hi - lo > 1) {
                const int64_t mid = (lo + hi) >> 1;
                if (item_off[mid] <= t0) lo = mid; else hi = mid;
            }
            s_q0 = lo;
            int64_t lo2 = lo, hi2 = q_hi;     // pairs starting before the tile's end
            const int64_t t1 = min(t_end, t0 + kGatherTile);
            while (hi2 - lo2 > 1) {
                const int64_t mid = (lo2 + hi2) >> 1;
                if (item_off[mid] < t1) lo2 = mid; else hi2 = mid;
            }
            s_n = (int)(lo2 - lo + 1);
        }
        __syncthreads();
        const int64_t q0 = s_q0;
        const int n = s_n;
        for (int u = threadIdx.x; u <= n; u += blockDim.x) s_off[u] = item_off[q0 + u];
        __syncthreads();
        for (int u = threadIdx.x; u < kGatherTile; u += blockDim.x) {
            const int64_t t = t0 + u;
            if (t >= t_end) break;
            int lo = 0, hi = n;    // pair: last j with s_off[j] <= t
            while (hi - lo > 1) {
                const int mid = (lo + hi) >> 1;
                if (s_off[mid] <= t) lo = mid; else hi = mid;
            }
            const int k = __ldg(list + q0 + lo);
            const int64_t e = __ldg(a_colptr + k) + (t - s_off[lo]);
            const int64_t b0 = __ldg(b_rowptr + k);
            const int rb = (int)(__ldg(b_rowptr + k + 1) - b0);
            const int64_t dst = __ldg(base + e);
            const float a = __ldg(a_val + e);
            for (int v = 0; 4 * v < rb; ++v) {
                int4 c4;
                float4 v4;
                load_b4(b_colidx + b0, b_val + b0, 4 * v, rb, c4, v4);
                store_run4(chat_col, chat_val, dst + 4 * v, c4, v4, a);
            }
        }
        __syncthreads();
    }
}

// nnz(a_*k) of the gather-list pairs (input of the item prefix scan)
__global__ void k_gather_item_counts(const int32_t *__restrict__ list, int64_t n, const int64_t *__restrict__ a_colptr,
                                     int64_t *__restrict__ cnt) {
    for (int64_t q = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; q < n; q += (int64_t)gridDim.x * blockDim.x) {
        const int k = list[q];
        cnt[q] = a_colptr[k + 1] - a_colptr[k];
    }
}

}  // namespace spg
