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
// Wide pieces (b_len >= 32): a warp holds a 128-entry chunk of the B sub-row in registers and
// streams it to every A entry of the piece (4 coalesced stores per lane and array).
// Thin pieces (b_len < 32): micro-blocks of w = 2^ceil(log2 b_len) lanes, 32/w A entries per
// warp step, so thin blocks do not idle lanes (block compaction, L406-L409 R).
__global__ void __launch_bounds__(kPieceThreads) k_expand_pieces(
    const Piece *__restrict__ pieces, const float *__restrict__ a_val, const int32_t *__restrict__ b_colidx,
    const float *__restrict__ b_val, const int64_t *__restrict__ base, int32_t *__restrict__ chat_col,
    float *__restrict__ chat_val) {
    __shared__ float s_a[kPieceAChunk];
    __shared__ int64_t s_dst[kPieceAChunk];
    const Piece pc = pieces[blockIdx.x];
    const int lane = lane_id(), w = warp_id();
    const int32_t *__restrict__ bc = b_colidx + pc.b_lo;
    const float *__restrict__ bv = b_val + pc.b_lo;
    for (int a0 = 0; a0 < pc.a_len; a0 += kPieceAChunk) {
        const int na = min(kPieceAChunk, pc.a_len - a0);
        for (int t = threadIdx.x; t < na; t += kPieceThreads) {
            s_a[t] = __ldg(a_val + pc.a_lo + a0 + t);
            s_dst[t] = __ldg(base + pc.a_lo + a0 + t) + pc.b_off;
        }
        __syncthreads();
        if (pc.b_len >= 32) {
            const int nchunks = (pc.b_len + 127) >> 7;
            const int slices = nchunks >= kPieceWarps ? 1 : kPieceWarps / nchunks;   // A slices per chunk
            for (int u = w; u < nchunks * slices; u += kPieceWarps) {
                const int c0 = (u / slices) << 7;
                const int sl = u % slices;
                int32_t cb[4];
                float vb[4];
#pragma unroll
                for (int q = 0; q < 4; ++q) {
                    const int j = c0 + q * 32 + lane;
                    cb[q] = j < pc.b_len ? __ldg(bc + j) : 0;
                    vb[q] = j < pc.b_len ? __ldg(bv + j) : 0.f;
                }
                const int lim = min(128, pc.b_len - c0);
                for (int a = sl; a < na; a += slices) {
                    const int64_t dst = s_dst[a] + c0;
                    const float av = s_a[a];
#pragma unroll
                    for (int q = 0; q < 4; ++q) {
                        const int j = q * 32 + lane;
                        if (j < lim) {
                            chat_col[dst + j] = cb[q];
                            chat_val[dst + j] = av * vb[q];
                        }
                    }
                }
            }
        } else {
            const int shift = ilog2_ceil((uint64_t)pc.b_len);
            const int mb = lane >> shift;
            const int sub = lane & ((1 << shift) - 1);
            const int g = 32 >> shift;
            const bool act = sub < pc.b_len;
            const int32_t cb = act ? __ldg(bc + sub) : 0;
            const float vb = act ? __ldg(bv + sub) : 0.f;
            if (act) {
                for (int a = w * g + mb; a < na; a += kPieceWarps * g) {
                    const int64_t dst = s_dst[a] + sub;
                    chat_col[dst] = cb;
                    chat_val[dst] = s_a[a] * vb;
                }
            }
        }
        __syncthreads();
    }
}

// B-Gathering (L369-L450): low performers with 2^(N-1) < nnz(b_k*) <= 2^N are packed
// 32/2^N per warp ("gathering factor 32/2^n", L438-L441 L); each micro-block of 2^N lanes
// keeps its B row in registers and loops over its A column, four entries per step with the
// (value, base) loads issued together.
template <int N>
__global__ void __launch_bounds__(256) k_expand_gathered(
    const int32_t *__restrict__ list, int64_t count, const int64_t *__restrict__ a_colptr,
    const float *__restrict__ a_val, const int64_t *__restrict__ b_rowptr, const int32_t *__restrict__ b_colidx,
    const float *__restrict__ b_val, const int64_t *__restrict__ base, int32_t *__restrict__ chat_col,
    float *__restrict__ chat_val) {
    constexpr int W = 1 << N;
    const int64_t slot = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> N;
    const int sub = threadIdx.x & (W - 1);
    if (slot >= count) return;
    const int k = __ldg(list + slot);
    const int64_t a0 = __ldg(a_colptr + k), a1 = __ldg(a_colptr + k + 1);
    const int64_t b0 = __ldg(b_rowptr + k);
    const int rb = (int)(__ldg(b_rowptr + k + 1) - b0);
    if (sub >= rb) return;
    const int32_t col = __ldg(b_colidx + b0 + sub);
    const float bv = __ldg(b_val + b0 + sub);
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
        for (int q = 0; q < 4; ++q) {
            chat_col[d[q] + sub] = col;
            chat_val[d[q] + sub] = av[q] * bv;
        }
    }
    for (; e < a1; ++e) {
        const int64_t d = __ldg(base + e) + sub;
        chat_col[d] = col;
        chat_val[d] = __ldg(a_val + e) * bv;
    }
}

}  // namespace spg
