// Stage (3): outer-product expansion into the row-bucketed intermediate matrix Ĉ.
//
// PAPER.md reconstructed Eq. (2) / Algorithm 1 (L150-L154, L325-L327 R): C = sum_k a_*k ⊗ b_k*;
// each product (i, j, a_ik*b_kj) is stored in Ĉ (L321-L323 L).  The row-wise offsets of
// stage (1) place every product of row i inside row i's bucket (L289-L291 R): the run of
// A entry e = (i, k) is Ĉ[base[e] .. base[e] + nnz(b_k*)), in B's (ascending) column order,
// padded with sentinel slots to a multiple of 8 (one 32-byte sector of columns and one of values, R16).
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
#ifndef SPG_EXP_PREFETCH
#define SPG_EXP_PREFETCH 0   // (A/B build knob: L2 prefetch of a tile's A values / run bases)
#endif
#ifndef SPG_EXP_TILE
#define SPG_EXP_TILE 2048
#endif
constexpr int kExpTile = SPG_EXP_TILE;   // units (16-byte vectors) per tile
constexpr int kExpUnroll = 4;
constexpr int kExpCtasPerSM = 3;   // 80 registers: 3 x 256 threads resident per SM, one persistent wave

// vectors of one run written by a block: the B sub-row rounded up to 8 slots (B tiles start on
// 8-slot boundaries, so the last tile of a row also writes the run's sentinel padding)
__device__ __forceinline__ int piece_nvec(const Piece &pc) { return (int)(pad_run(pc.b_len) >> 2); }

__global__ void k_piece_units(const Piece *__restrict__ pieces, int64_t n, int64_t *__restrict__ units) {
    for (int64_t q = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; q < n; q += (int64_t)gridDim.x * blockDim.x) {
        const Piece pc = pieces[q];
        units[q] = (int64_t)pc.a_len * piece_nvec(pc);
    }
}

// B' = B with every row padded to a multiple of kRunAlign slots (col = INT32_MAX, val = 0), 16-byte
// stores.  Lane per row for rows of <= 64 entries; the warp's longer rows (hub rows of thousands
// of entries) are then copied by the whole warp, one after another (a thread per row alone left
// AB18's 100K-entry rows on one thread: 1.2 ms).
__device__ __forceinline__ void pad_b_vec(const int32_t *__restrict__ b_colidx, const float *__restrict__ b_val,
                                          int64_t b0, int64_t rb, int64_t d0, int64_t j, int32_t *__restrict__ bp_col,
                                          float *__restrict__ bp_val) {
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

__global__ void k_pad_b(const int64_t *__restrict__ b_rowptr, const int32_t *__restrict__ b_colidx,
                        const float *__restrict__ b_val, int64_t K, int32_t *__restrict__ bp_col,
                        float *__restrict__ bp_val) {
    const int lane = threadIdx.x & 31;
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t kb = (int64_t)blockIdx.x * blockDim.x + (threadIdx.x & ~31); kb < K; kb += stride) {
        const int64_t k = kb + lane;
        int64_t b0 = 0, rb = 0;
        if (k < K) { b0 = b_rowptr[k]; rb = b_rowptr[k + 1] - b0; }
        const bool lng = rb > 64;
        if (!lng)
            for (int64_t j = 0; j < pad_run(rb); j += 4) pad_b_vec(b_colidx, b_val, b0, rb, bp_start(b0, k), j, bp_col, bp_val);
        unsigned m = __ballot_sync(0xffffffffu, lng);
        while (m) {
            const int l = __ffs(m) - 1;
            m &= m - 1;
            const int64_t kl = kb + l;
            const int64_t bl = __shfl_sync(0xffffffffu, b0, l), rl = __shfl_sync(0xffffffffu, rb, l);
            for (int64_t j = 4 * lane; j < pad_run(rl); j += 128) pad_b_vec(b_colidx, b_val, bl, rl, bp_start(bl, kl), j, bp_col, bp_val);
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

// r / nv for r < 2^22 in fp32 with an exact fix-up (else the 64-bit division)
__device__ __forceinline__ int64_t div_units(int64_t r, int nv) {
    if (r < (1 << 22)) {
        const int ri = (int)r;
        int ai = __float2int_rz(((float)ri + 0.5f) / (float)nv);
        ai -= (ai * nv > ri);
        ai += ((ai + 1) * nv <= ri);
        return ai;
    }
    return r / nv;   // (huge unsplit blocks: enable_split = 0)
}

// Pieces overlapping one tile are staged in shared memory (unit offset, A start, B' source,
// vectors per run, B offset), so a unit's only global loads are its A value / run base and its
// B' vector -- all independent, one memory round trip -- followed by the two 16-byte stores.
// A tile overlapping more than kExpPieceCache blocks (only gathered 1-unit blocks can do that)
// searches the block list in global memory instead.
constexpr int kExpPieceCache = 1024;

__global__ void __launch_bounds__(kExpThreads) k_expand_flat(
    const Piece *__restrict__ pieces, const int64_t *__restrict__ uoff, int64_t npieces,
    const int64_t *__restrict__ tile_p0, const int64_t *__restrict__ b_rowptr, const int32_t *__restrict__ bp_col,
    const float *__restrict__ bp_val, const float *__restrict__ a_val, const int64_t *__restrict__ base,
    int32_t *__restrict__ chat_col, float *__restrict__ chat_val, unsigned long long *lbi,
    const int64_t *__restrict__ unit_lo_ptr) {
    lbi_start(lbi);
    __shared__ int64_t s_uoff[kExpPieceCache + 1];
    __shared__ int64_t s_alo[kExpPieceCache];
    __shared__ int64_t s_bsrc[kExpPieceCache];
    __shared__ int32_t s_nv[kExpPieceCache];
    __shared__ int32_t s_boff[kExpPieceCache];
    const int64_t total = uoff[npieces];
    const int64_t ntiles = (total + kExpTile - 1) / kExpTile;
    const int64_t unit_lo = *unit_lo_ptr;        // (units below unit_lo: the block kernel's)
    const int64_t tile0 = unit_lo / kExpTile;
    for (int64_t tile = tile0 + blockIdx.x; tile < ntiles; tile += gridDim.x) {
        const int64_t f0 = max(unit_lo, tile * kExpTile), f1 = min(total, tile * kExpTile + kExpTile);
        const int64_t p0 = tile_p0[tile];
        const int64_t pend = tile_p0[tile + 1] + 1;   // blocks [p0, pend) overlap the tile
        const int np = (int)min(pend - p0, (int64_t)kExpPieceCache + 1);
        const bool cached = np <= kExpPieceCache;
        __syncthreads();                               // previous tile's readers are done
        if (cached) {
            for (int q = threadIdx.x; q < np; q += kExpThreads) {
                const Piece pc = pieces[p0 + q];
                s_uoff[q] = uoff[p0 + q];
                s_alo[q] = pc.a_lo;
                s_bsrc[q] = bp_start(b_rowptr[pc.k], pc.k) + pc.b_off;
                s_nv[q] = piece_nvec(pc);
                s_boff[q] = pc.b_off;
            }
            if (threadIdx.x == 0) s_uoff[np] = INT64_MAX;
        }
        __syncthreads();
#if SPG_EXP_PREFETCH
        if (cached) {   // L2 prefetch of the A values / run bases the tile's units will load
            for (int q = threadIdx.x; q < np; q += kExpThreads) {
                const int64_t u0 = max(s_uoff[q], f0) - s_uoff[q], u1 = min(s_uoff[q + 1], f1) - s_uoff[q];
                if (u1 <= u0) continue;
                const int nv = s_nv[q];
                const int64_t e0 = s_alo[q] + u0 / nv, e1 = s_alo[q] + (u1 - 1) / nv;
                for (int64_t e = e0 & ~(int64_t)15; e <= e1; e += 16)   // 128-byte lines of base[]
                    asm volatile("prefetch.global.L2 [%0];" ::"l"(base + e));
                for (int64_t e = e0 & ~(int64_t)31; e <= e1; e += 32)   // ... of a_val[]
                    asm volatile("prefetch.global.L2 [%0];" ::"l"(a_val + e));
                if (SPG_EXP_PREFETCH >= 2)   // ... and of the block's B' row (columns, values)
                    for (int64_t j = s_bsrc[q] & ~(int64_t)31; j < s_bsrc[q] + 4 * nv; j += 32) {
                        asm volatile("prefetch.global.L2 [%0];" ::"l"(bp_col + j));
                        asm volatile("prefetch.global.L2 [%0];" ::"l"(bp_val + j));
                    }
            }
        }
#endif
        // kExpUnroll units per thread per step, their loads issued together
        int pj = 0;             // cached: local block index (never decreases)
        int64_t gj = p0;        // uncached: global block index
        for (int64_t fb = f0 + threadIdx.x; fb < f1; fb += kExpUnroll * kExpThreads) {
            int64_t dst[kExpUnroll];
            float av[kExpUnroll];
            int4 c4[kExpUnroll];
            float4 w4[kExpUnroll];
            bool ok[kExpUnroll];
#pragma unroll
            for (int u = 0; u < kExpUnroll; ++u) {
                const int64_t f = fb + u * kExpThreads;
                ok[u] = f < f1;
                if (!ok[u]) continue;
                int64_t alo, bsrc, uo;
                int nv, boff;
                if (cached) {
                    int hi = np;                   // last block with s_uoff <= f
                    while (hi - pj > 1) {
                        const int mid = (pj + hi) >> 1;
                        if (s_uoff[mid] <= f) pj = mid; else hi = mid;
                    }
                    uo = s_uoff[pj]; alo = s_alo[pj]; bsrc = s_bsrc[pj]; nv = s_nv[pj]; boff = s_boff[pj];
                } else {
                    int64_t hi = pend;
                    while (hi - gj > 1) {
                        const int64_t mid = (gj + hi) >> 1;
                        if (__ldg(uoff + mid) <= f) gj = mid; else hi = mid;
                    }
                    const Piece pc = pieces[gj];
                    uo = __ldg(uoff + gj); alo = pc.a_lo; bsrc = bp_start(__ldg(b_rowptr + pc.k), pc.k) + pc.b_off;
                    nv = piece_nvec(pc); boff = pc.b_off;
                }
                const int64_t r = f - uo;
                const int64_t a = div_units(r, nv);
                const int v = (int)(r - a * nv);
                const int64_t e = alo + a;
                av[u] = __ldg(a_val + e);
                dst[u] = __ldg(base + e) + boff + 4 * v;
                c4[u] = __ldg(reinterpret_cast<const int4 *>(bp_col + bsrc + 4 * v));
                w4[u] = __ldg(reinterpret_cast<const float4 *>(bp_val + bsrc + 4 * v));
            }
#pragma unroll
            for (int u = 0; u < kExpUnroll; ++u)
                if (ok[u]) {
                    // streaming (evict-first) stores: Ĉ is written once and read by the merge much
                    // later, so it should not push B' (re-read by every A entry of k) out of L2
                    __stcs(reinterpret_cast<int4 *>(chat_col + dst[u]), c4[u]);
                    __stcs(reinterpret_cast<float4 *>(chat_val + dst[u]),
                           make_float4(av[u] * w4[u].x, av[u] * w4[u].y, av[u] * w4[u].z, av[u] * w4[u].w));
                }
        }
    }
    lbi_end(lbi);
}

// ------------------------------------------------ block path: TMA-staged B' tiles -------
// Split pieces and whole Normal blocks (>= 32 effective threads, L317-L318 R): one block at a
// time per CTA, claimed in order.  The block's B' tile (nv 16-byte vectors of columns and of
// values, <= 1024 each) is brought into shared memory by two bulk copies (cp.async.bulk, TMA
// engine; double-buffered: the next block's tile streams in while this one is written), then
// every A entry e of the block is written as one run Ĉ[base[e] + b_off ..) = (cols, a_e * vals):
// groups of W = min(32, 2^ceil(log2 nv)) lanes take an A entry each and stride over its vectors
// -- two 16-byte stores per 4 products, no per-unit search, division or global B' load.
#ifndef EXP_BLK_VEC
#define EXP_BLK_VEC 512
#endif
constexpr int kExpBlkThreads = 256;
constexpr int kExpBlkVec = EXP_BLK_VEC;   // vectors of one B' buffer (longer B tiles: sub-tiles)
constexpr int kExpBlkSmem = 2 * 2 * kExpBlkVec * 16;   // 2 buffers x (cols, vals) = 64 KB

__device__ __forceinline__ void exp_mbar_init(uint64_t *mbar) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"((uint32_t)__cvta_generic_to_shared(mbar)), "r"(1)
                 : "memory");
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void exp_bulk_load(void *dst, const void *src, uint32_t bytes, uint64_t *mbar) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                     (uint32_t)__cvta_generic_to_shared(dst)),
                 "l"(src), "r"(bytes), "r"((uint32_t)__cvta_generic_to_shared(mbar))
                 : "memory");
}
__device__ __forceinline__ void exp_expect_tx(uint64_t *mbar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(
                     (uint32_t)__cvta_generic_to_shared(mbar)),
                 "r"(bytes)
                 : "memory");
}
__device__ __forceinline__ void exp_wait(uint64_t *mbar, uint32_t parity) {
    asm volatile(
        "{\n"
        ".reg .pred p;\n"
        "WAIT_%=:\n"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
        "@!p bra WAIT_%=;\n"
        "}\n" ::"r"((uint32_t)__cvta_generic_to_shared(mbar)),
        "r"(parity)
        : "memory");
}

__global__ void __launch_bounds__(kExpBlkThreads) k_expand_blocks(
    const Piece *__restrict__ pieces, int64_t nblk, const int64_t *__restrict__ b_rowptr,
    const int32_t *__restrict__ bp_col, const float *__restrict__ bp_val, const float *__restrict__ a_val,
    const int64_t *__restrict__ base, int32_t *__restrict__ chat_col, float *__restrict__ chat_val,
    unsigned long long *ticket, unsigned long long *lbi) {
    lbi_start(lbi);
    extern __shared__ __align__(16) unsigned char smem_raw[];
    __shared__ uint64_t mbar[2];
    __shared__ int64_t s_next;
    __shared__ float s_av[kExpBlkThreads];      // the block's A values and run bases (a_len <= 256:
    __shared__ int64_t s_dst[kExpBlkThreads];   //  split_ca_max bounds every block's A range)
    const int tid = threadIdx.x;
    if (tid == 0) {
        exp_mbar_init(&mbar[0]);
        exp_mbar_init(&mbar[1]);
    }
    __syncthreads();
    uint32_t phases = 0;   // mbarrier parity of buffer b in bit b
    // issue the bulk copies of vectors [v0, v0 + min(rest, kExpBlkVec)) of block q into buffer b
    auto issue = [&](int64_t q, int b, int v0) {
        const Piece pc = pieces[q];
        const int nv = min(piece_nvec(pc) - v0, kExpBlkVec);
        const int64_t src = bp_start(b_rowptr[pc.k], pc.k) + pc.b_off + 4 * (int64_t)v0;
        int4 *dc = reinterpret_cast<int4 *>(smem_raw + (size_t)b * 2 * kExpBlkVec * 16);
        float4 *dv = reinterpret_cast<float4 *>(dc + kExpBlkVec);
        exp_expect_tx(&mbar[b], (uint32_t)nv * 32u);
        exp_bulk_load(dc, bp_col + src, (uint32_t)nv * 16u, &mbar[b]);
        exp_bulk_load(dv, bp_val + src, (uint32_t)nv * 16u, &mbar[b]);
    };
    int64_t cur = 0;
    if (tid == 0) {
        cur = (int64_t)atomicAdd(ticket, 1ull);
        if (cur < nblk) issue(cur, 0, 0);
        s_next = cur;
    }
    __syncthreads();
    cur = s_next;
    int b = 0;
    while (cur < nblk) {
        __syncthreads();   // (s_next of the previous round read; the other buffer's readers done)
        if (tid == 0) {    // prefetch the next block into the other buffer
            const int64_t nx = (int64_t)atomicAdd(ticket, 1ull);
            if (nx < nblk) issue(nx, b ^ 1, 0);
            s_next = nx;
        }
        const Piece pc = pieces[cur];
        const int nvall = piece_nvec(pc);

        const int4 *sc = reinterpret_cast<const int4 *>(smem_raw + (size_t)b * 2 * kExpBlkVec * 16);
        const float4 *sv = reinterpret_cast<const float4 *>(sc + kExpBlkVec);
        // (a whole Normal block's B row can exceed one buffer: its further sub-tiles reuse this one)
        for (int v0 = 0; v0 < nvall; v0 += kExpBlkVec) {
            if (v0 > 0) {
                __syncthreads();   // the previous sub-tile's readers are done
                if (tid == 0) {
                    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
                    issue(cur, b, v0);
                }
            }
            exp_wait(&mbar[b], (phases >> b) & 1u);
            phases ^= 1u << b;
            const int nv = min(nvall - v0, kExpBlkVec);
            const int lw = nv >= 32 ? 5 : (nv <= 1 ? 0 : 32 - __clz(nv - 1));   // lanes per A entry: 2^lw
            const int W = 1 << lw;
            const int sub = tid >> lw;                          // entry slot of this lane group
            const int nsub = kExpBlkThreads >> lw;
            const int li = tid & (W - 1);
            for (int a0 = 0; a0 < pc.a_len; a0 += kExpBlkThreads) {   // A entries in chunks of 256
                const int na = min(pc.a_len - a0, kExpBlkThreads);
                __syncthreads();   // (the previous chunk's readers are done)
                if (tid < na) {    // one coalesced load per A entry
                    s_av[tid] = __ldg(a_val + pc.a_lo + a0 + tid);
                    s_dst[tid] = __ldg(base + pc.a_lo + a0 + tid) + pc.b_off;
                }
                __syncthreads();
                for (int a = sub; a < na; a += nsub) {
                    const float av = s_av[a];
                    const int64_t dst = s_dst[a] + 4 * (int64_t)v0;
                    int4 *oc = reinterpret_cast<int4 *>(chat_col + dst);
                    float4 *ov = reinterpret_cast<float4 *>(chat_val + dst);
                    for (int v = li; v < nv; v += W) {
                        const float4 w = sv[v];
                        __stcs(oc + v, sc[v]);
                        __stcs(ov + v, make_float4(av * w.x, av * w.y, av * w.z, av * w.w));
                    }
                }
            }
        }
        __syncthreads();
        if (tid == 0) asm volatile("fence.proxy.async.shared::cta;" ::: "memory");   // before the next prefetch
        cur = s_next;
        b ^= 1;
    }
    lbi_end(lbi);
}

// ------------------------------------------------ row-product expansion (comparison) ---
// The paper's comparison point (row-product / Gustavson order, L476-L478 R): the same Ĉ (every
// run at base[e]) written row by row -- one warp per row of A walks the row's entries (A in CSR
// order, built by a counting sort of the CSC entries) and copies nnz(b_k*) scaled B' vectors per
// entry.  No Block Reorganizer: a row's work is one warp's, whatever its size.  Selected by
// options.reserved[3] = 1 (bench --opt reserved... / tests); DESIGN.md §5 compares the two.
__global__ void k_row_entries(const int64_t *__restrict__ a_colptr, int64_t K, int64_t nnz_a,
                              const int32_t *__restrict__ a_rowidx, const int64_t *__restrict__ b_rowptr,
                              const int64_t *__restrict__ rptr, unsigned *__restrict__ cursor,
                              int64_t *__restrict__ list_e, int32_t *__restrict__ list_k) {
    int64_t e0 = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) * 8;
    if (e0 >= nnz_a) return;
    int64_t k = upper_bound_idx(a_colptr, 0, K, e0);
    int64_t kend = __ldg(a_colptr + k + 1);
    for (int64_t e = e0; e < e0 + 8 && e < nnz_a; ++e) {
        while (e >= kend) { ++k; kend = __ldg(a_colptr + k + 1); }
        if (__ldg(b_rowptr + k + 1) > __ldg(b_rowptr + k)) {
            const int i = a_rowidx[e];
            const int64_t q = rptr[i] + atomicAdd(cursor + i, 1u);
            list_e[q] = e;
            list_k[q] = (int32_t)k;
        }
    }
}

__global__ void __launch_bounds__(256) k_expand_rows(const int64_t *__restrict__ rptr, int64_t M,
                                                     const int64_t *__restrict__ list_e,
                                                     const int32_t *__restrict__ list_k,
                                                     const int64_t *__restrict__ b_rowptr,
                                                     const int32_t *__restrict__ bp_col,
                                                     const float *__restrict__ bp_val,
                                                     const float *__restrict__ a_val,
                                                     const int64_t *__restrict__ base, int32_t *__restrict__ chat_col,
                                                     float *__restrict__ chat_val) {
    const int lane = lane_id();
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t i = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; i < M; i += nw) {
        const int64_t e_lo = rptr[i], e_hi = rptr[i + 1];
        for (int64_t c0 = e_lo; c0 < e_hi; c0 += 32) {
            const int64_t q = c0 + lane;
            int nv = 0;
            int64_t src = 0, dst = 0;
            float av = 0.f;
            if (q < e_hi) {
                const int64_t e = list_e[q];
                const int32_t k = list_k[q];
                const int64_t b0 = __ldg(b_rowptr + k);
                nv = (int)(pad_run(__ldg(b_rowptr + k + 1) - b0) >> 2);
                src = bp_start(b0, k);
                dst = base[e];
                av = a_val[e];
            }
            const int inc = warp_incl_sum(nv);
            const int off = inc - nv, tot = __shfl_sync(0xffffffffu, inc, 31);
            for (int u0 = 0; u0 < tot; u0 += 32) {
                const int u = u0 + lane;
                int j = 0;               // owner lane: number of lanes with inc <= u
#pragma unroll
                for (int step = 16; step > 0; step >>= 1) {
                    const int probe = __shfl_sync(0xffffffffu, inc, min(j + step - 1, 31));
                    if (j + step <= 32 && probe <= u) j += step;
                }
                j = min(j, 31);
                const int64_t s_j = __shfl_sync(0xffffffffu, src, j), d_j = __shfl_sync(0xffffffffu, dst, j);
                const float a_j = __shfl_sync(0xffffffffu, av, j);
                const int v = u - __shfl_sync(0xffffffffu, off, j);
                if (u < tot) {
                    const int4 c4 = __ldg(reinterpret_cast<const int4 *>(bp_col + s_j + 4 * v));
                    const float4 w4 = __ldg(reinterpret_cast<const float4 *>(bp_val + s_j + 4 * v));
                    __stcs(reinterpret_cast<int4 *>(chat_col + d_j + 4 * v), c4);
                    __stcs(reinterpret_cast<float4 *>(chat_val + d_j + 4 * v),
                           make_float4(a_j * w4.x, a_j * w4.y, a_j * w4.z, a_j * w4.w));
                }
            }
        }
    }
}

}  // namespace spg
