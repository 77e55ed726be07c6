// Stage (3): outer-product expansion into the row-bucketed intermediate matrix Ĉ.
//
// PAPER.md reconstructed Eq. (2) / Algorithm 1 (L150-L154, L325-L327 R): C = sum_k a_*k ⊗ b_k*;
// each product (i, j, a_ik*b_kj) is stored in Ĉ (L321-L323 L).  The row-wise offsets of
// stage (1) place every product of row i inside row i's bucket (L289-L291 R): the run of
// A entry e = (i, k) is Ĉ[base[e] .. base[e] + nnz(b_k*)), in B's (ascending) column order.
//
// Ĉ layout: SoA, row implicit: chat_col int32[nnz(Ĉ)], chat_val fp32[nnz(Ĉ)] (8 B/product).
#pragma once
#include "analysis.cuh"

namespace spg {

constexpr int kPieceThreads = 128;

// B-Split pieces and whole blocks (Normal pairs).  One CTA per piece.  The paper's block has
// nnz(b_k*) effective threads, each looping over the A column (L385-L386 R, L411-L415 L);
// here a micro-block of w = min(32, 2^ceil(log2 b_len)) lanes covers the B sub-row and the
// 32/w micro-blocks of a warp take different A entries of the same piece, so thin pieces do
// not idle lanes (block compaction, L406-L409 R).
__global__ void __launch_bounds__(kPieceThreads) k_expand_pieces(
    const Piece *__restrict__ pieces, const float *__restrict__ a_val, const int32_t *__restrict__ b_colidx,
    const float *__restrict__ b_val, const int64_t *__restrict__ base, int32_t *__restrict__ chat_col,
    float *__restrict__ chat_val) {
    const Piece pc = pieces[blockIdx.x];
    const int shift = pc.b_len >= 32 ? 5 : ilog2_ceil((uint64_t)pc.b_len);
    const int w = 1 << shift;
    const int g = 32 >> shift;
    const int mb = lane_id() >> shift;
    const int sub = lane_id() & (w - 1);
    const int slots = (kPieceThreads / 32) * g;
    const int32_t *__restrict__ bc = b_colidx + pc.b_lo;
    const float *__restrict__ bv = b_val + pc.b_lo;
    for (int ai = warp_id() * g + mb; ai < pc.a_len; ai += slots) {
        const int64_t e = pc.a_lo + ai;
        const float a = __ldg(a_val + e);
        const int64_t dst = __ldg(base + e) + pc.b_off;
        for (int j = sub; j < pc.b_len; j += w) {
            chat_col[dst + j] = __ldg(bc + j);
            chat_val[dst + j] = a * __ldg(bv + j);
        }
    }
}

// B-Gathering (L369-L450): low performers with 2^(N-1) < nnz(b_k*) <= 2^N are packed
// 32/2^N per warp ("gathering factor 32/2^n", L438-L441 L); each micro-block of 2^N lanes
// keeps its B row in registers and loops over its A column.
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
    const bool act = sub < rb;
    const int32_t col = act ? __ldg(b_colidx + b0 + sub) : 0;
    const float bv = act ? __ldg(b_val + b0 + sub) : 0.f;
    if (!act) return;
    for (int64_t e = a0; e < a1; ++e) {
        const int64_t dst = __ldg(base + e) + sub;
        chat_col[dst] = col;
        chat_val[dst] = __ldg(a_val + e) * bv;
    }
}

}  // namespace spg
