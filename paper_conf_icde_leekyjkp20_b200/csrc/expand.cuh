// Stage (3): outer-product expansion into the row-bucketed intermediate matrix Ĉ.
//
// PAPER.md reconstructed Eq. (2) / Algorithm 1 (L150-L154, L325-L327 R): C = sum_k a_*k ⊗ b_k*;
// each product (i, j, a_ik*b_kj) is stored in Ĉ (L321-L323 L).  The row-wise offsets of
// stage (1) place every product of row i inside row i's bucket (L289-L291 R): the run of
// A entry e = (i, k) is Ĉ[base[e] .. base[e] + nnz(b_k*)), in B's (ascending) column order,
// padded with sentinel slots to a multiple of 4 (16 bytes).
//
// Ĉ layout: SoA, row implicit: chat_col int32[nnz(Ĉ)], chat_val fp32[nnz(Ĉ)] (8 B/product).
//
// Blackwell mapping of the Block Reorganizer's blocks.  Every expansion block -- a B-Split piece
// of a Dominator (L320-L415), a whole Normal block, or a Low-performer block -- is a rectangle
// (A entries [a_lo, a_lo + a_len)) x (B entries [b_lo, b_lo + b_len)).  Its work is cut into
// units of one 16-byte vector (4 products) of one run, and the blocks are laid end to end in
// unit space (prefix uoff[] over the block list: Split pieces, Normal blocks, then the
// Low-performer blocks in B-Gathering order).  A persistent grid walks fixed tiles of
// kExpTile units, so a tile holds a part of one big piece or many gathered low performers
// packed together -- the paper's B-Gathering of underloaded blocks into one thread block
// (L369-L412 R) with one lane per 4 effective threads -- and no thread idles on a thin block
// (the micro-block compaction of L406-L409 R).  The store-bound inner step is: A value and run
// base (L1-cached, shared by the nv units of a run), one 16-byte B vector from the padded copy
// B' (16-byte aligned rows, sentinel-filled), 4 products, two 16-byte stores; consecutive
// threads write consecutive vectors of a run.
#pragma once
#include "analysis.cuh"

namespace spg {

constexpr int kExpThreads = 256;
constexpr int kExpTile = 2048;   // units (16-byte vectors) per tile
constexpr int kExpUnroll = 4;
constexpr int kExpCtasPerSM = 3;   // 80 registers: 3 x 256 threads resident per SM, one persistent wave

// vectors of one run written by a block: the B sub-row rounded up to 4 slots (B tiles start on
// 4-slot boundaries, so the last tile of a row also writes the run's sentinel padding)
__device__ __forceinline__ int piece_nvec(const Piece &pc) { return (pc.b_len + 3) >> 2; }

__global__ void k_piece_units(const Piece *__restrict__ pieces, int64_t n, int64_t *__restrict__ units) {
    for (int64_t q = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; q < n; q += (int64_t)gridDim.x * blockDim.x) {
        const Piece pc = pieces[q];
        units[q] = (int64_t)pc.a_len * piece_nvec(pc);
    }
}

// B' = B with every row padded to a multiple of 4 slots (col = INT32_MAX, val = 0); one thread
// per row (rows are short), 16-byte stores
__global__ void k_pad_b(const int64_t *__restrict__ b_rowptr, const int32_t *__restrict__ b_colidx,
                        const float *__restrict__ b_val, int64_t K, const int64_t *__restrict__ b_prow,
                        int32_t *__restrict__ bp_col, float *__restrict__ bp_val) {
    for (int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; k < K; k += (int64_t)gridDim.x * blockDim.x) {
        const int64_t b0 = b_rowptr[k], rb = b_rowptr[k + 1] - b0;
        const int64_t d0 = b_prow[k];
        for (int64_t j = 0; j < rb; j += 4) {
            int32_t c[4];
            float v[4];
#pragma unroll
            for (int u = 0; u < 4; ++u) {
                c[u] = j + u < rb ? b_colidx[b0 + j + u] : 0x7fffffff;
                v[u] = j + u < rb ? b_val[b0 + j + u] : 0.f;
            }
            *reinterpret_cast<int4 *>(bp_col + d0 + j) = make_int4(c[0], c[1], c[2], c[3]);
            *reinterpret_cast<float4 *>(bp_val + d0 + j) = make_float4(v[0], v[1], v[2], v[3]);
        }
    }
}

// first block of every tile: tile_p0[t] = last p with uoff[p] <= t * kExpTile (t <= ntiles)
__global__ void k_tile_first_piece(const int64_t *__restrict__ uoff, int64_t npieces, int64_t ntiles,
                                   int64_t *__restrict__ tile_p0) {
    for (int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; t <= ntiles; t += (int64_t)gridDim.x * blockDim.x) {
        const int64_t f = min(t * kExpTile, uoff[npieces] - 1);
        int64_t lo = 0, hi = npieces;
        while (hi - lo > 1) {
            const int64_t mid = (lo + hi) >> 1;
            if (uoff[mid] <= f) lo = mid; else hi = mid;
        }
        tile_p0[t] = lo;
    }
}

__global__ void __launch_bounds__(kExpThreads) k_expand_flat(
    const Piece *__restrict__ pieces, const int64_t *__restrict__ uoff, int64_t npieces,
    const int64_t *__restrict__ tile_p0, const int64_t *__restrict__ b_prow, const int32_t *__restrict__ bp_col,
    const float *__restrict__ bp_val, const float *__restrict__ a_val, const int64_t *__restrict__ base,
    int32_t *__restrict__ chat_col, float *__restrict__ chat_val) {
    const int64_t total = uoff[npieces];
    const int64_t ntiles = (total + kExpTile - 1) / kExpTile;
    for (int64_t tile = blockIdx.x; tile < ntiles; tile += gridDim.x) {
        const int64_t f0 = tile * kExpTile, f1 = min(total, f0 + kExpTile);
        const int64_t p0 = tile_p0[tile];
        const int64_t pend = tile_p0[tile + 1] + 1;   // blocks [p0, pend) overlap the tile
        // kExpUnroll units per thread per step, their loads issued together (memory-level
        // parallelism: each unit is a short chain block -> A entry -> B vector -> store)
        int64_t pj = p0;
        for (int64_t fb = f0 + threadIdx.x; fb < f1; fb += kExpUnroll * kExpThreads) {
            int64_t dst[kExpUnroll], src[kExpUnroll];
            float av[kExpUnroll];
            bool ok[kExpUnroll];
#pragma unroll
            for (int u = 0; u < kExpUnroll; ++u) {
                const int64_t f = fb + u * kExpThreads;
                ok[u] = f < f1;
                if (!ok[u]) continue;
                int64_t hi = pend;                 // last block with uoff <= f (never decreases)
                while (hi - pj > 1) {
                    const int64_t mid = (pj + hi) >> 1;
                    if (__ldg(uoff + mid) <= f) pj = mid; else hi = mid;
                }
                const Piece pc = pieces[pj];
                const int nv = piece_nvec(pc);
                const int64_t r = f - __ldg(uoff + pj);
                int64_t a;
                if (r < (1 << 22)) {               // r / nv in fp32, then an exact fix-up
                    const int ri = (int)r;
                    int ai = __float2int_rz(((float)ri + 0.5f) / (float)nv);
                    ai -= (ai * nv > ri);
                    ai += ((ai + 1) * nv <= ri);
                    a = ai;
                } else {                           // (huge unsplit blocks: enable_split = 0)
                    a = r / nv;
                }
                const int v = (int)(r - a * nv);
                const int64_t e = pc.a_lo + a;
                av[u] = __ldg(a_val + e);
                dst[u] = __ldg(base + e) + pc.b_off + 4 * v;
                src[u] = __ldg(b_prow + pc.k) + pc.b_off + 4 * v;
            }
            int4 c4[kExpUnroll];
            float4 w4[kExpUnroll];
#pragma unroll
            for (int u = 0; u < kExpUnroll; ++u)
                if (ok[u]) {
                    c4[u] = __ldg(reinterpret_cast<const int4 *>(bp_col + src[u]));
                    w4[u] = __ldg(reinterpret_cast<const float4 *>(bp_val + src[u]));
                }
#pragma unroll
            for (int u = 0; u < kExpUnroll; ++u)
                if (ok[u]) {
                    *reinterpret_cast<int4 *>(chat_col + dst[u]) = c4[u];
                    *reinterpret_cast<float4 *>(chat_val + dst[u]) =
                        make_float4(av[u] * w4[u].x, av[u] * w4[u].y, av[u] * w4[u].z, av[u] * w4[u].w);
                }
        }
    }
}

}  // namespace spg
