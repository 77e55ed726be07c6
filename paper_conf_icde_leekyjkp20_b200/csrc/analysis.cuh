// Stage (1) workload analysis and stage (2) categorisation / Block Reorganizer lists.
//
// (1) PAPER.md §IV-B L326-L330 L + L289-L291 R: "Block reorganizer first calculates nnz(Ĉ)
//     ... There are two different ways to compute memory space ... The row-wise nnz is used
//     to relocate the outer-product's elements with same row closer together ... We also
//     calculate the block-wise nnz for workload classification."
// (2) L304-L318 R (Dominator / Low performer), L320-L415 (B-Splitting), L369-L450
//     (B-Gathering), L452-L477 L (B-Limiting rows).  B200 readings R1-R8: DESIGN.md §2.
#pragma once
#include "common.cuh"

namespace spg {

// pair classes (spgemm_inspect SPGEMM_VIEW_PAIR_CLASS) -- the paper's categories
enum : int8_t { PC_EMPTY = 0, PC_DOMINATOR = 1, PC_NORMAL = 2, PC_LOW = 3 };
// pair processing buckets: 0 split pieces, 1 single-piece blocks, 2 + n*16 + c gathered, 98 none
constexpr int kPairBucketSplit = 0;
constexpr int kPairBucketPiece = 1;
constexpr int kPairBucketGather0 = 2;
constexpr int kPairBucketEmpty = 98;
constexpr int kNumPairBuckets = 99;
// row processing classes (SPGEMM_VIEW_ROW_CLASS) and buckets
enum : int8_t { RC_EMPTY = 0, RC_PASS = 1, RC_WARP = 2, RC_WARP_SORT = 3, RC_GROUP_SORT = 4, RC_LIMITED = 5 };
constexpr int kRowBucketPass = 0;
constexpr int kRowBucketWarp = 1;      // cap <= 32: register bitonic, 1 slot per lane
constexpr int kRowBucketWarp64 = 2;    // cap <= 64 / 128 / 256: register bitonic, 2 / 4 / 8 slots per lane
constexpr int kRowBucketWarp128 = 3;
constexpr int kRowBucketSort256 = 4;
constexpr int kRowBucketSort512 = 5;   // cap <= 512 / 1K / 2K / 4K: bucket sort, 2 / 4 / 8 / 16 warps
constexpr int kRowBucketSort1K = 6;
constexpr int kRowBucketSort2K = 7;
constexpr int kRowBucketSort4K = 8;
constexpr int kRowBucketLim0 = 9;      // 9 + (39 - floor(log2 L)): longest rows first
constexpr int kRowBucketEmpty = 49;
constexpr int kNumRowBuckets = 50;
constexpr int kWarpRowMax = 32;
// Ĉ runs are padded to multiples of kRunAlign slots (32 B: one DRAM sector of columns and one of
// values) with sentinel entries (col = INT32_MAX, val = 0), so that every run starts 16-byte
// aligned (vector stores, bulk copies) and no 32-byte sector is shared by two runs -- two runs of
// a row are written by different blocks at different times, and a sector written half by each
// used to cost a read-modify-write in DRAM (R16).
constexpr int kRunAlign = 8;
__host__ __device__ __forceinline__ int64_t pad_run(int64_t x) { return (x + kRunAlign - 1) & ~(int64_t)(kRunAlign - 1); }
constexpr int kSort256Max = 256;
constexpr int kSort512Max = 512;
constexpr int kSort1KMax = 1024;
constexpr int kSort2KMax = 2048;
constexpr int64_t kLimitCapacity = 4096;   // largest bucket length of the non-limited merge bins
constexpr int kUnitRowMax = 2048;          // short rows (merged by the unit kernel): padded bucket <= this

struct PlanScalars {
    unsigned long long nnz_chat;     // sum_k work[k]
    unsigned long long k_nonempty;   // #pairs with work > 0
    unsigned long long m_nonempty;   // #rows with rowwork > 0
    unsigned long long max_rowwork;
    unsigned long long max_deg;      // max runs (A entries with nnz(b_k*) > 0) in a row
    unsigned long long rowwise_sum;  // sum_i rowwork[i] (nnz(Ĉ) counted row-wise)
    unsigned long long lim_runs;     // sum of runs over limited rows
    unsigned long long lim_max_deg;  // max runs of a limited row
    unsigned long long lim_max_L;    // max products of a limited row
    unsigned long long long_slots;   // padded Ĉ slots of the long rows (side buffer of the merge)
    unsigned long long lim_slots;    // padded Ĉ slots of the limited rows (column-group scratch)
    int invalid;                     // validation failure bits
    int pad;
};

struct Piece {          // one expansion block: A entries [a_lo, a_lo+a_len) x B entries [b_lo, b_lo+b_len)
    int64_t a_lo;
    int64_t b_lo;
    int32_t a_len;
    int32_t b_len;
    int32_t b_off;      // b_lo - rowptr_B[k]: offset of the B sub-row inside each product run
    int32_t k;
};

// ---------------------------------------------------------------- validation (optional) ---
__global__ void k_validate_ptr(const int64_t *__restrict__ ptr, int64_t nseg, int64_t nnz, int *flag, int bit) {
    int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i == 0 && (ptr[0] != 0 || ptr[nseg] != nnz)) atomicOr(flag, bit);
    if (i < nseg && ptr[i + 1] < ptr[i]) atomicOr(flag, bit);
}

// entries of segment s are idx[ptr[s]..ptr[s+1]); each thread walks 8 consecutive entries.
__global__ void k_validate_idx(const int64_t *__restrict__ ptr, const int32_t *__restrict__ idx, int64_t nseg,
                               int64_t nnz, int64_t bound, int *flag, int bit) {
    int64_t e0 = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) * 8;
    if (e0 >= nnz) return;
    int64_t s = upper_bound_idx(ptr, 0, nseg, e0);
    bool bad = false;
    for (int64_t e = e0; e < e0 + 8 && e < nnz; ++e) {
        while (__ldg(ptr + s + 1) <= e) ++s;
        int32_t v = idx[e];
        if (v < 0 || v >= bound) bad = true;
        if (e > __ldg(ptr + s) && idx[e - 1] >= v) bad = true;
    }
    if (bad) atomicOr(flag, bit);
}

// ---------------------------------------------------------------- row window -------------
// spgemm_plan_rows: rows [r0, r1) of A (CSC, rows ascending per column) are, in every column, one
// contiguous range of entries -- found by two binary searches; the window's A' is those ranges
// packed (row indices minus r0), so C' = A' x B is rows [r0, r1) of C.
__global__ void k_window_count(const int64_t *__restrict__ colptr, const int32_t *__restrict__ rowidx, int64_t K,
                               int32_t r0, int32_t r1, int64_t *__restrict__ lo, int64_t *__restrict__ cnt) {
    for (int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; k < K; k += (int64_t)gridDim.x * blockDim.x) {
        const int64_t a = colptr[k], b = colptr[k + 1];
        int64_t l = a, h = b;   // first entry with row >= r0
        while (l < h) { const int64_t m = (l + h) >> 1; if (rowidx[m] < r0) l = m + 1; else h = m; }
        const int64_t first = l;
        h = b;                  // first entry with row >= r1
        while (l < h) { const int64_t m = (l + h) >> 1; if (rowidx[m] < r1) l = m + 1; else h = m; }
        lo[k] = first;
        cnt[k] = l - first;
    }
}

// one warp per column copies its window range
__global__ void k_window_copy(const int64_t *__restrict__ lo, const int64_t *__restrict__ newptr, int64_t K,
                              const int32_t *__restrict__ rowidx, const float *__restrict__ val, int32_t r0,
                              int32_t *__restrict__ out_idx, float *__restrict__ out_val) {
    const int lane = threadIdx.x & 31;
    for (int64_t k = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; k < K;
         k += ((int64_t)gridDim.x * blockDim.x) >> 5) {
        const int64_t src = lo[k], dst = newptr[k], n = newptr[k + 1] - dst;
        for (int64_t q = lane; q < n; q += 32) {
            out_idx[dst + q] = rowidx[src + q] - r0;
            out_val[dst + q] = val[src + q];
        }
    }
}

// ---------------------------------------------------------------- stage (1) --------------
// Block-wise nnz: work[k] = nnz(a_*k) * nnz(b_k*)  (L326-L330 L, L290-L291 R).
__global__ void __launch_bounds__(256) k_pair_work(const int64_t *__restrict__ a_colptr,
                                                   const int64_t *__restrict__ b_rowptr, int64_t K,
                                                   int64_t *__restrict__ work, PlanScalars *sc) {
    __shared__ unsigned long long sm[2][8];
    unsigned long long s = 0, ne = 0;
    for (int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; k < K; k += (int64_t)gridDim.x * blockDim.x) {
        int64_t w = (a_colptr[k + 1] - a_colptr[k]) * (b_rowptr[k + 1] - b_rowptr[k]);
        work[k] = w;
        s += (unsigned long long)w;
        ne += w > 0;
    }
    s = warp_sum(s);
    ne = warp_sum(ne);
    if (lane_id() == 0) { sm[0][warp_id()] = s; sm[1][warp_id()] = ne; }
    __syncthreads();
    if (threadIdx.x == 0) {
        unsigned long long a = 0, b = 0;
        for (int w = 0; w < 8; ++w) { a += sm[0][w]; b += sm[1][w]; }
        atomicAdd(&sc->nnz_chat, a);
        atomicAdd(&sc->k_nonempty, b);
    }
}

// Row-wise nnz: rowwork[i] += nnz(b_k*) for every stored a_ik; deg[i] = #runs of Ĉ row i.
// Each thread walks 8 consecutive A entries (column found once by binary search).
__global__ void __launch_bounds__(256) k_row_work(const int64_t *__restrict__ a_colptr,
                                                  const int32_t *__restrict__ a_rowidx, int64_t K, int64_t nnz_a,
                                                  const int64_t *__restrict__ b_rowptr,
                                                  unsigned long long *__restrict__ rowwork, int32_t *__restrict__ deg,
                                                  unsigned long long *__restrict__ rowcap) {
    int64_t e0 = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) * 8;
    if (e0 >= nnz_a) return;
    int64_t k = upper_bound_idx(a_colptr, 0, K, e0);
    int64_t kend = __ldg(a_colptr + k + 1);
    int64_t rb = __ldg(b_rowptr + k + 1) - __ldg(b_rowptr + k);
    for (int64_t e = e0; e < e0 + 8 && e < nnz_a; ++e) {
        while (e >= kend) {
            ++k;
            kend = __ldg(a_colptr + k + 1);
            rb = __ldg(b_rowptr + k + 1) - __ldg(b_rowptr + k);
        }
        if (rb > 0) {
            int32_t i = a_rowidx[e];
            atomicAdd(rowwork + i, (unsigned long long)rb);
            atomicAdd(deg + i, 1);
            if (rowcap) atomicAdd(rowcap + i, (unsigned long long)pad_run(rb));
        }
    }
}

__global__ void __launch_bounds__(256) k_row_reduce(const int64_t *__restrict__ rowwork,
                                                    const int32_t *__restrict__ deg, int64_t M, PlanScalars *sc) {
    __shared__ unsigned long long sm[4][8];
    unsigned long long ne = 0, mx = 0, md = 0, sum = 0;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < M; i += (int64_t)gridDim.x * blockDim.x) {
        int64_t w = rowwork[i];
        sum += (unsigned long long)w;
        ne += w > 0;
        mx = max(mx, (unsigned long long)w);
        md = max(md, (unsigned long long)deg[i]);
    }
    ne = warp_sum(ne);
    sum = warp_sum(sum);
    mx = warp_max(mx);
    md = warp_max(md);
    if (lane_id() == 0) { sm[0][warp_id()] = ne; sm[1][warp_id()] = mx; sm[2][warp_id()] = md; sm[3][warp_id()] = sum; }
    __syncthreads();
    if (threadIdx.x == 0) {
        unsigned long long a = 0, b = 0, c = 0, d = 0;
        for (int w = 0; w < 8; ++w) { a += sm[0][w]; b = max(b, sm[1][w]); c = max(c, sm[2][w]); d += sm[3][w]; }
        atomicAdd(&sc->rowwise_sum, d);
        atomicAdd(&sc->m_nonempty, a);
        atomicMax(&sc->max_rowwork, b);
        atomicMax(&sc->max_deg, c);
    }
}

// Run bases: the run of products of A entry e = (i, k) occupies Ĉ positions
// [base[e], base[e] + nnz(b_k*)) inside row i's bucket (cursor starts at rowoff[i]), followed
// by pad_run(nnz(b_k*)) - nnz(b_k*) sentinel slots.
// rows whose padded Ĉ bucket is longer than this get the plan's column range (bucket-sort bins)
constexpr int64_t kRangeMinSlots = 256;

__global__ void __launch_bounds__(256) k_run_base(const int64_t *__restrict__ a_colptr,
                                                  const int32_t *__restrict__ a_rowidx, int64_t K, int64_t nnz_a,
                                                  const int64_t *__restrict__ b_rowptr,
                                                  unsigned long long *__restrict__ cursor, int64_t *__restrict__ base,
                                                  const int64_t *__restrict__ rowoff = nullptr,
                                                  const int32_t *__restrict__ b_colidx = nullptr,
                                                  int32_t *__restrict__ rowmn = nullptr,
                                                  int32_t *__restrict__ rowmx = nullptr) {
    // rowmn / rowmx (optional): the exact column range of row i of C -- min / max over the stored
    // a_ik of b_k*'s first / last column (B's rows are ascending): every product of the row is in
    // it and its ends are attained, so the bucket-sort bins need no range reduction.  Only rows
    // whose padded bucket exceeds kRangeMinSlots (the bucket-sorted ones) pay the two atomics.
    int64_t e0 = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) * 8;
    if (e0 >= nnz_a) return;
    int64_t k = upper_bound_idx(a_colptr, 0, K, e0);
    int64_t kend = __ldg(a_colptr + k + 1);
    int64_t rb0 = __ldg(b_rowptr + k), rb1 = __ldg(b_rowptr + k + 1);
    for (int64_t e = e0; e < e0 + 8 && e < nnz_a; ++e) {
        while (e >= kend) {
            ++k;
            kend = __ldg(a_colptr + k + 1);
            rb0 = rb1;
            rb1 = __ldg(b_rowptr + k + 1);
        }
        const int64_t rb = rb1 - rb0;
        if (rb > 0) {
            const int32_t i = a_rowidx[e];
            base[e] = (int64_t)atomicAdd(cursor + i, (unsigned long long)pad_run(rb));
            if (rowmn && __ldg(rowoff + i + 1) - __ldg(rowoff + i) > kRangeMinSlots) {
                atomicMin(rowmn + i, __ldg(b_colidx + rb0));
                atomicMax(rowmx + i, __ldg(b_colidx + rb1 - 1));
            }
        } else {
            base[e] = -1;
        }
    }
}

// r_p = first row i with rowoff[i] >= floor(p * total / parts)  (lower bound), p = 1..parts-1
__global__ void k_partition_bounds(const int64_t *__restrict__ rowoff, int64_t M, int parts, int64_t *__restrict__ bounds) {
    int p = blockIdx.x * blockDim.x + threadIdx.x;
    if (p > parts) return;
    if (p == 0) { bounds[0] = 0; return; }
    if (p == parts) { bounds[parts] = M; return; }
    const int64_t total = rowoff[M];
    const unsigned __int128 t128 = (unsigned __int128)p * (unsigned __int128)total;
    const int64_t target = (int64_t)(t128 / (unsigned)parts);
    int64_t lo = 0, hi = M + 1;   // first index in [0, M] with rowoff[idx] >= target
    while (lo < hi) {
        int64_t mid = (lo + hi) >> 1;
        if (rowoff[mid] < target) lo = mid + 1; else hi = mid;
    }
    bounds[p] = min(lo, M);
}

// ---------------------------------------------------------------- stage (2) --------------
struct SplitParams {
    int64_t piece_work;
    int32_t b_tile;
    int32_t split_ca_max;
    int32_t fixed_f;      // > 0: every Dominator split by this factor (Fig. 11 sweep; capped at ca's)
};

// Splitting factor f = 2^n (L410-L413 L): smallest power of two whose greedy chunk of
// ceil(ca/f) column entries keeps a piece within piece_work products and split_ca_max
// computations per thread.  A fixed factor (options.reserved[7], the Fig. 11 sweep) is used as
// given, but never beyond the smallest power of two >= ca (one entry per piece).
__device__ __forceinline__ int64_t splitting_factor(int64_t ca, int64_t blen, const SplitParams &p) {
    if (p.fixed_f > 0) {
        int64_t f = 1;
        while (f < p.fixed_f && f < ca) f <<= 1;
        return f;
    }
    int64_t f = 1;
    while (f < ca) {
        int64_t chunk = (ca + f - 1) / f;
        if (chunk * blen <= p.piece_work && chunk <= p.split_ca_max) break;
        f <<= 1;
    }
    return f;
}

struct ClassifyParams {
    int64_t t_dom;
    int32_t split_ca_max;
    int32_t enable_split;
    int32_t enable_gather;
};

// Dominator: block-wise nnz > threshold (L309-L311 R) or nnz(a_*k) > split_ca_max (R3);
// Low performer: < 32 effective threads nnz(b_k*) (L317-L318 R); Normal otherwise.
__global__ void __launch_bounds__(256) k_pair_classify(const int64_t *__restrict__ a_colptr,
                                                       const int64_t *__restrict__ b_rowptr,
                                                       const int64_t *__restrict__ work, int64_t K, ClassifyParams p,
                                                       SplitParams sp, int8_t *__restrict__ cls,
                                                       uint8_t *__restrict__ bucket, int64_t *__restrict__ npieces) {
    for (int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; k < K; k += (int64_t)gridDim.x * blockDim.x) {
        int64_t ca = a_colptr[k + 1] - a_colptr[k];
        int64_t rb = b_rowptr[k + 1] - b_rowptr[k];
        int64_t w = work[k];
        int8_t c;
        int b;
        if (w == 0) {
            c = PC_EMPTY;
            b = kPairBucketEmpty;
        } else if (w > p.t_dom || ca > p.split_ca_max) {
            c = PC_DOMINATOR;
            b = p.enable_split ? kPairBucketSplit : kPairBucketPiece;
        } else if (rb < kWarp) {
            c = PC_LOW;
            if (p.enable_gather) {
                int n = ilog2_ceil((uint64_t)rb);              // 2^(n-1) < rb <= 2^n  (L438-L439 L)
                int cc = min(15, ilog2_floor((uint64_t)ca));   // per-thread loop length class (R5)
                b = kPairBucketGather0 + n * 16 + cc;
            } else {
                b = kPairBucketPiece;
            }
        } else {
            c = PC_NORMAL;
            b = kPairBucketPiece;
        }
        cls[k] = c;
        bucket[k] = (uint8_t)b;
        int64_t np = 0;
        if (b == kPairBucketSplit) {   // B-Splitting piece count (pieces are laid out in ascending k)
            const int64_t blen = min(rb, (int64_t)sp.b_tile);
            const int64_t f = splitting_factor(ca, blen, sp);
            const int64_t chunk = (ca + f - 1) / f;
            np = ((ca + chunk - 1) / chunk) * ((rb + sp.b_tile - 1) / sp.b_tile);
        }
        npieces[k] = np;
    }
}

// Pieces of dominator d in order (B tile t, A piece q); one warp per dominator.
__global__ void k_piece_fill(const int32_t *__restrict__ dom, int64_t ndom, const int64_t *__restrict__ a_colptr,
                             const int64_t *__restrict__ b_rowptr, SplitParams p,
                             const int64_t *__restrict__ piece_off, Piece *__restrict__ pieces) {
    int64_t d = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    if (d >= ndom) return;
    int k = dom[d];
    int64_t a0 = a_colptr[k], ca = a_colptr[k + 1] - a0;
    int64_t b0 = b_rowptr[k], rb = b_rowptr[k + 1] - b0;
    int64_t blen = min(rb, (int64_t)p.b_tile);
    int64_t f = splitting_factor(ca, blen, p);
    int64_t chunk = (ca + f - 1) / f;
    int64_t npa = (ca + chunk - 1) / chunk;
    int64_t nb = (rb + p.b_tile - 1) / p.b_tile;
    int64_t base = piece_off[k];
    for (int64_t q = lane_id(); q < npa * nb; q += 32) {
        int64_t t = q / npa, a = q % npa;
        Piece pc;
        pc.a_lo = a0 + a * chunk;
        pc.a_len = (int32_t)min(chunk, ca - a * chunk);
        pc.b_off = (int32_t)(t * p.b_tile);
        pc.b_lo = b0 + pc.b_off;
        pc.b_len = (int32_t)min((int64_t)p.b_tile, rb - t * p.b_tile);
        pc.k = k;
        pieces[base + q] = pc;
    }
}

// One piece per non-split block (Normal pairs; also Low performers when B-Gathering is off
// and Dominators when B-Splitting is off: the paper's plain one-block-per-pair mapping).
__global__ void k_piece_whole(const int32_t *__restrict__ list, int64_t n, const int64_t *__restrict__ a_colptr,
                              const int64_t *__restrict__ b_rowptr, Piece *__restrict__ pieces) {
    for (int64_t q = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; q < n; q += (int64_t)gridDim.x * blockDim.x) {
        int k = list[q];
        Piece pc;
        pc.a_lo = a_colptr[k];
        pc.a_len = (int32_t)(a_colptr[k + 1] - pc.a_lo);
        pc.b_lo = b_rowptr[k];
        pc.b_len = (int32_t)(b_rowptr[k + 1] - pc.b_lo);
        pc.b_off = 0;
        pc.k = k;
        pieces[q] = pc;
    }
}

// B' (B with rows padded to kRunAlign = 8 slots, R16) row k starts at bp_start(b_rowptr[k], k) =
// b_rowptr[k] + 15k rounded up to 8 slots: 32-byte aligned and clear of row k + 1 (row k ends by
// b_rowptr[k+1] + 15k + 14) without a scan over the padded lengths; B' holds nnz(B) + 15K + 8 slots.
__host__ __device__ __forceinline__ int64_t bp_start(int64_t rp, int64_t k) {
    return (rp + (2 * kRunAlign - 1) * k + kRunAlign - 1) & ~(int64_t)(kRunAlign - 1);
}

// Merge row classes.  Limited rows (L > t_lim, L452-L477 L) get B-Limited merge blocks;
// a row made of a single run (one A entry) is already sorted and duplicate-free.
__global__ void __launch_bounds__(256) k_row_classify(const int64_t *__restrict__ rowwork,
                                                      const int64_t *__restrict__ rowoff,
                                                      const int32_t *__restrict__ deg, int64_t M, int64_t t_lim,
                                                      int64_t cap_max, int8_t *__restrict__ rcls,
                                                      uint8_t *__restrict__ bucket, PlanScalars *sc) {
    __shared__ unsigned long long sm[5][8];
    unsigned long long runs = 0, mdeg = 0, mlen = 0, lslots = 0, limslots = 0;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < M; i += (int64_t)gridDim.x * blockDim.x) {
        // L = products of the row (paper class); cap = its padded bucket length (kernel capacity)
        const int64_t L = rowwork[i];
        const int64_t cap = rowoff[i + 1] - rowoff[i];
        int8_t c;
        int b;
        if (L == 0) { c = RC_EMPTY; b = kRowBucketEmpty; }
        else if (deg[i] == 1 && cap <= kUnitRowMax) { c = RC_PASS; b = kRowBucketPass; }
        else if (L > t_lim || cap > cap_max) {
            c = RC_LIMITED;
            b = kRowBucketLim0 + (39 - min(39, ilog2_floor((uint64_t)L)));
            runs += (unsigned long long)deg[i];
            mdeg = max(mdeg, (unsigned long long)deg[i]);
            mlen = max(mlen, (unsigned long long)cap);
            limslots += (unsigned long long)cap;
        }
        else if (cap <= kWarpRowMax) { c = RC_WARP; b = kRowBucketWarp; }
        else if (cap <= 64) { c = RC_WARP_SORT; b = kRowBucketWarp64; }
        else if (cap <= 128) { c = RC_WARP_SORT; b = kRowBucketWarp128; }
        else if (cap <= kSort256Max) { c = RC_WARP_SORT; b = kRowBucketSort256; }
        else if (cap <= kSort512Max) { c = RC_WARP_SORT; b = kRowBucketSort512; }
        else if (cap <= kSort1KMax) { c = RC_WARP_SORT; b = kRowBucketSort1K; }
        else if (cap <= kSort2KMax) { c = RC_GROUP_SORT; b = kRowBucketSort2K; }
        else { c = RC_GROUP_SORT; b = kRowBucketSort4K; }
        rcls[i] = c;
        bucket[i] = (uint8_t)b;
        if (cap > kUnitRowMax || c == RC_LIMITED) lslots += (unsigned long long)cap;   // long row (side buffer)
    }
    runs = warp_sum(runs);
    mdeg = warp_max(mdeg);
    mlen = warp_max(mlen);
    lslots = warp_sum(lslots);
    limslots = warp_sum(limslots);
    if (lane_id() == 0) {
        sm[0][warp_id()] = runs; sm[1][warp_id()] = mdeg; sm[2][warp_id()] = mlen; sm[3][warp_id()] = lslots;
        sm[4][warp_id()] = limslots;
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        unsigned long long a = 0, b = 0, c = 0, d = 0, e = 0;
        for (int w = 0; w < 8; ++w) {
            a += sm[0][w]; b = max(b, sm[1][w]); c = max(c, sm[2][w]); d += sm[3][w]; e += sm[4][w];
        }
        if (d) atomicAdd(&sc->long_slots, d);
        if (e) atomicAdd(&sc->lim_slots, e);
        if (a) atomicAdd(&sc->lim_runs, a);
        if (b) atomicMax(&sc->lim_max_deg, b);
        if (c) atomicMax(&sc->lim_max_L, c);
    }
}

// bucket starts: out[b] = offs[b * ntiles] for b < nb, out[nb] = offs[nb * ntiles] (= n)
__global__ void k_bucket_starts(const int64_t *__restrict__ offs, int nb, int64_t ntiles, int64_t *__restrict__ out) {
    int b = blockIdx.x * blockDim.x + threadIdx.x;
    if (b <= nb) out[b] = offs[(int64_t)b * ntiles];
}

// Limited rows: index map and run lists (base, length) of their products.
__global__ void k_lim_index(const int32_t *__restrict__ rows, int64_t nlim, const int32_t *__restrict__ deg,
                            int32_t *__restrict__ lim_index, int64_t *__restrict__ nruns) {
    for (int64_t q = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; q < nlim; q += (int64_t)gridDim.x * blockDim.x) {
        int r = rows[q];
        lim_index[r] = (int32_t)q;
        nruns[q] = deg[r];
    }
}

__global__ void __launch_bounds__(256) k_lim_runs(const int64_t *__restrict__ a_colptr,
                                                  const int32_t *__restrict__ a_rowidx, int64_t K, int64_t nnz_a,
                                                  const int64_t *__restrict__ b_rowptr,
                                                  const int64_t *__restrict__ base, const int32_t *__restrict__ lim_index,
                                                  const int64_t *__restrict__ run_start, int32_t *__restrict__ run_fill,
                                                  int64_t *__restrict__ run_base, int32_t *__restrict__ run_len) {
    int64_t e0 = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) * 8;
    if (e0 >= nnz_a) return;
    int64_t k = upper_bound_idx(a_colptr, 0, K, e0);
    int64_t kend = __ldg(a_colptr + k + 1);
    for (int64_t e = e0; e < e0 + 8 && e < nnz_a; ++e) {
        while (e >= kend) { ++k; kend = __ldg(a_colptr + k + 1); }
        int32_t li = lim_index[a_rowidx[e]];
        int64_t b = base[e];
        if (li >= 0 && b >= 0) {
            int slot = atomicAdd(run_fill + li, 1);
            run_base[run_start[li] + slot] = b;
            run_len[run_start[li] + slot] = (int32_t)(__ldg(b_rowptr + k + 1) - __ldg(b_rowptr + k));
        }
    }
}

}  // namespace spg
