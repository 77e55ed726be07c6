// Stage (4) merge of the short rows into C, fused with C's placement (no compaction pass).
//
// PAPER.md §IV-D L452-L455 L: "elements with the same indices are merged into unique elements";
// BASELINE.json north_star: "a row-bucketed sort plus segmented reduce into CSR".
//
// B200 design ("merge tiles"):
//   * A *tile* is a run of consecutive short rows (padded Ĉ slots <= kTileCap in total, at most
//     kTileThreads rows), packed greedily in row order, or one chunk of a B-Limited row (merged
//     beforehand in place by the long-row kernels of merge.cuh) that only has to move.
//   * One persistent kernel claims tiles in row order (atomic ticket).  Per short tile:
//       1. one thread issues two bulk copies (cp.async.bulk, TMA engine) of the tile's keys and
//          values into shared memory (mbarrier completion); the other threads load the row table;
//       2. every thread takes kTileEPT consecutive slots into registers; per-row column min / max
//          by shared atomics (one per row segment of a thread);
//       3. row r gets nb_r = 2^ceil(log2 Lv_r) buckets over its column span, bucket =
//          base_r + ((col - min_r) >> sh_r); the tile's buckets are row-major, so one histogram
//          (shared atomics; the returned count is the key's rank in its bucket) and one scan order
//          the whole tile by (row, column bucket);
//       4. keys of single-key buckets and of exact buckets (sh_r = 0: every key equal) land at
//          their final slot; the others rank against the keys of their bucket (equal keys by
//          scatter position) and move after a barrier (in place: one buffer);
//       5. fp64 segmented reduction over contiguous slices (a segment ends at a key change or a
//          row start) into a staging copy of the merged tile, in shared memory;
//       6. decoupled look-back over the tiles' merged counts gives the tile's output offset P;
//          C's row pointers and the merged rows are written at [P, P + U) -- in place in the Ĉ
//          arrays, which is safe because every tile reads its input before it publishes its
//          count and writes its output only after all its predecessors have published (the
//          output of tile t lies below the end of tile t's input).
//   * A long-row chunk tile reads its slice of the merged row (registers), publishes its length,
//     resolves P and writes it (same protocol: memmove-safe).
#pragma once
#include "merge.cuh"

namespace spg {

constexpr int kTileThreads = 512;
constexpr int kTileEPT = 8;
constexpr int kTileCap = kTileThreads * kTileEPT;   // 4096 slots (= kLimitCapacity: longer rows are B-Limited)
constexpr int kTileMaxRows = kTileThreads;          // rows of one tile (every row owns >= 1 thread)
constexpr int kTileRowChunk = 1024;                 // rows per warp of the tile-table builder
constexpr int kCopyChunk = kTileThreads * 8;        // merged entries per long-row chunk tile
static_assert(kTileCap >= kLimitCapacity, "every non-limited row must fit one tile");

constexpr int kGroupCap = kTileCap - 8;             // products of one long-row group tile (merge_long.cuh)

// Tile kinds (one persistent kernel walks them in row order):
//   TK_ROWS   rows [x, y) of Ĉ (short rows)
//   TK_GROUP  group x of a long row (merge_long.cuh): sorted + reduced like a row; y = the row when
//             it is the row's first group (C row pointer), else -1
//   TK_COPY   chunk y of the merged entries of dense group x (merged by k_long_dense, scratch);
//             z = the row when it starts the row, else -1
//   TK_INPLACE chunk y of long row x merged in place at the head of its Ĉ bucket (legacy long-row
//             kernels of merge.cuh)
enum : int32_t { TK_ROWS = 0, TK_GROUP = 1, TK_COPY = 2, TK_INPLACE = 3 };
struct TileDesc {
    int32_t kind, x, y, z;
};

// long-row group tables (merge_long.cuh) seen by the tile-table builder and the tile kernel
struct LongTables {
    const int32_t *lim_index;   // row -> limited-list entry (or -1)
    const int64_t *yoff;        // first group of list entry q
    const int32_t *g_num;       // groups of list entry q
    const int64_t *g_off;       // scratch offset of a group
    const int32_t *g_cnt;       // products (sort groups) / merged entries (merged dense groups)
    const int8_t *g_kind;
};

// ---- tile table ------------------------------------------------------------------------------
// Rows [c*kTileRowChunk, (c+1)*kTileRowChunk) are packed by warp c, greedily in row order (tiles never
// cross a chunk boundary): the lanes load 32 consecutive rows at a time and the warp closes a tile at
// the first lane whose row no longer fits (prefix sums + ballot), so a step costs one round of
// shuffles instead of a dependent load per row.  Pass 1 counts the tiles of every chunk, pass 2
// writes them; a B-Limited row closes the open tile and emits its own tiles (one lane loops).
template <bool FILL>
__global__ void __launch_bounds__(128) k_tile_table(const int64_t *__restrict__ rowoff, const int8_t *__restrict__ rcls,
                                                    const int64_t *__restrict__ ccount, LongTables lt, int64_t M,
                                                    int64_t *__restrict__ count, const int64_t *__restrict__ base,
                                                    TileDesc *__restrict__ tiles) {
    const int64_t c = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int lane = lane_id();
    const int64_t i0 = c * kTileRowChunk;
    if (i0 >= M) return;
    const int64_t i1 = min(M, i0 + kTileRowChunk);
    int64_t nt = 0, o = FILL ? base[c] : 0;   // (warp-uniform)
    int64_t open = -1;                        // first row of the open short tile
    int64_t acc = 0;                          // its slots
    for (int64_t w0 = i0; w0 < i1; w0 += 32) {
        const int64_t i = w0 + lane;
        const bool in = i < i1;
        const int64_t cap = in ? rowoff[i + 1] - rowoff[i] : 0;
        const bool lim = in && rcls[i] == RC_LIMITED;
        int done = 0;
        const int nin = i1 - w0 < 32 ? (int)(i1 - w0) : 32;
        while (done < nin) {
            // rows [done, j) join the open tile; lane j is a B-Limited row or does not fit
            // a short row owns ceil(cap / EPT) threads of the tile (>= its slots / EPT); a tile has T
            const int64_t cc = (lane >= done && lane < nin) ? (cap + kTileEPT - 1) / kTileEPT : 0;
            const int64_t pre = warp_incl_sum(cc);
            const int64_t first = open >= 0 ? open : w0 + done;   // first row of the tile being grown
            const bool ev = lane >= done && lane < nin &&
                            (lim || acc + pre > kTileThreads || (w0 + lane) - first >= kTileMaxRows);
            const unsigned m = __ballot_sync(kFull, ev);
            const int j = m ? __ffs(m) - 1 : nin;
            if (j > done) {
                if (open < 0) { open = w0 + done; acc = 0; }
                acc += __shfl_sync(kFull, pre, j - 1);
            }
            if (j >= nin) break;
            const bool limj = __shfl_sync(kFull, lim, j);
            if (open >= 0) {   // close the open tile before row w0 + j
                if (FILL && lane == 0) tiles[o] = TileDesc{TK_ROWS, (int32_t)open, (int32_t)(w0 + j), 0};
                ++o;
                ++nt;
                open = -1;
                acc = 0;
            }
            if (limj) {
                const int64_t r = w0 + j;
                int64_t emitted = 0;
                if (lane == 0) {
                    auto emit = [&](int32_t kind, int32_t x, int32_t y, int32_t z) {
                        if (FILL) tiles[o + emitted] = TileDesc{kind, x, y, z};
                        ++emitted;
                    };
                    if (lt.g_num) {   // column groups (merge_long.cuh)
                        const int32_t q = lt.lim_index[r];
                        const int32_t G = lt.g_num[q];
                        const int64_t Y = lt.yoff[q];
                        for (int32_t g = 0; g < G; ++g) {
                            const int64_t gi = Y + g;
                            if (lt.g_kind[gi] == 0) {   // GK_SORT
                                emit(TK_GROUP, (int32_t)gi, g == 0 ? (int32_t)r : -1, 0);
                            } else {
                                const int32_t U = lt.g_cnt[gi];
                                const int32_t nch = U > kCopyChunk ? (U + kCopyChunk - 1) / kCopyChunk : 1;
                                for (int32_t q2 = 0; q2 < nch; ++q2)
                                    emit(TK_COPY, (int32_t)gi, q2, (g == 0 && q2 == 0) ? (int32_t)r : -1);
                            }
                        }
                    } else {          // merged in place (legacy long-row kernels)
                        const int64_t U = ccount[r];
                        const int64_t nch = U > kCopyChunk ? (U + kCopyChunk - 1) / kCopyChunk : 1;
                        for (int64_t q2 = 0; q2 < nch; ++q2) emit(TK_INPLACE, (int32_t)r, (int32_t)q2, 0);
                    }
                }
                emitted = __shfl_sync(kFull, emitted, 0);
                o += emitted;
                nt += emitted;
                done = j + 1;
            } else {
                open = w0 + j;   // row j starts the next tile
                acc = (__shfl_sync(kFull, cap, j) + kTileEPT - 1) / kTileEPT;
                done = j + 1;
            }
        }
    }
    if (open >= 0) {
        if (FILL && lane == 0) tiles[o] = TileDesc{TK_ROWS, (int32_t)open, (int32_t)i1, 0};
        ++nt;
    }
    if (!FILL && lane == 0) count[c] = nt;
}

// ---- bulk copies (TMA engine) and mbarriers ---------------------------------------------------
__device__ __forceinline__ uint32_t smem_u32(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }

__device__ __forceinline__ void mbar_init(uint64_t *mbar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(mbar)), "r"(count) : "memory");
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t *mbar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(mbar)), "r"(bytes)
                 : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t *mbar, uint32_t parity) {
    asm volatile(
        "{\n"
        ".reg .pred p;\n"
        "WAIT_%=:\n"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
        "@!p bra WAIT_%=;\n"
        "}\n" ::"r"(smem_u32(mbar)),
        "r"(parity)
        : "memory");
}
// generic-proxy accesses of shared memory before this point are ordered before later bulk copies
__device__ __forceinline__ void fence_proxy_async_smem() {
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}
// global -> shared bulk copy of `bytes` (multiple of 16, both addresses 16-byte aligned)
__device__ __forceinline__ void bulk_g2s(void *dst, const void *src, uint32_t bytes, uint64_t *mbar) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                     smem_u32(dst)),
                 "l"(src), "r"(bytes), "r"(smem_u32(mbar))
                 : "memory");
}

// ---- the tile kernel ------------------------------------------------------------------------
struct TileArgs {
    const TileDesc *tiles;
    const int64_t *ntiles;         // device scalar
    const int64_t *rowoff;         // padded Ĉ offsets [M + 1]
    const int64_t *rowwork;        // products per row
    const int64_t *ccount;         // merged length of the B-Limited rows (merged in place)
    int32_t *col;                  // in: Ĉ; out: C's columns at [0, nnz(C))
    float *val;
    int64_t *crowptr;              // out: C row pointers [M + 1]
    int64_t M;
    unsigned long long *status;    // look-back words [#tiles], zeroed
    unsigned long long *ticket;    // zeroed
    LongTables lt;                 // long-row groups (merge_long.cuh)
    int32_t *scol;                 // their scratch
    float *sval;
    int debug;                     // options.reserved[1] (tuning only): 1 = no look-back (every tile
                                   // writes at its own input position: wrong C, timing only), 2 =
                                   // per-phase clock64 totals of thread 0 into prof[0..16)
    unsigned long long *prof;
};
#define TILE_PH(k)                                                   \
    do {                                                             \
        if (prof_on) {                                               \
            const long long _t = clock64();                          \
            ph[k] += (unsigned long long)(_t - t_last);              \
            t_last = _t;                                             \
        }                                                            \
    } while (0)

template <int T, int EPT>
struct TileSmem {
    static constexpr int kCap = T * EPT;
    static constexpr int kNb = 2 * kCap;   // row r's buckets live at [2 ro[r], 2 ro[r] + 2^ceil(log2 Lv)) < 2 ro[r+1]
    static constexpr int kRowWords = 7 * (kTileMaxRows + 1);
    // layout: keys | vals (bulk copy target, scatter target, then the merged tile) | hist (bucket counts /
    // starts, then the sorted tile) | binfo (bucket of every scattered slot, then slice carries) | rows
    static constexpr int kBytes = kCap * 8 + (kNb + 8) * 4 + kCap * 4 + kRowWords * 4;
    static_assert(kNb >= 2 * kCap && kCap >= 3 * T, "sorted tile aliases the histogram, carries binfo");
};

// exclusive sum over the CTA with one barrier: `sc` holds NW + 1 ints and must not be written again
// before a later barrier (callers alternate two buffers)
template <int NW>
__device__ __forceinline__ int cta_excl_sum(int v, int *sc, int *total) {
    const int inc = warp_incl_sum(v);
    const int w = warp_id();
    if (lane_id() == 31) sc[w] = inc;
    __syncthreads();
    const int t = lane_id() < NW ? sc[lane_id()] : 0;
    const int ci = warp_incl_sum(t);
    *total = __shfl_sync(kFull, ci, NW - 1);
    return __shfl_sync(kFull, ci - t, w) + inc - v;
}

// bucket parameters of a row: as many buckets as fit its region of the histogram (2 cap slots, cap =
// the row's padded slots >= its products), i.e. 2^floor(log2(2 cap)), over its column span [mn, mx]
__device__ __forceinline__ int row_shift(int cap, int mn, int mx) {
    const uint32_t span = (uint32_t)(mx - mn);
    const int bits = span ? 32 - __clz(span) : 0;
    return max(0, bits - (32 - __clz(2 * cap) - 1));
}

template <int T, int EPT>
__global__ void __launch_bounds__(T, 2) k_merge_tiles(TileArgs a) {
    using S = TileSmem<T, EPT>;
    constexpr int NW = T / 32;
    constexpr int RW = kTileMaxRows + 1;
    constexpr int BPT = S::kNb / T;                    // buckets per thread in the scan
    static_assert(EPT % 4 == 0 && BPT % 4 == 0, "vector accesses");
    constexpr int E2M = (S::kCap + T - 1) / T + 1;    // max slice length of the reduction (odd stride)
    extern __shared__ __align__(16) unsigned char smem_raw[];
    int32_t *sk = (int32_t *)smem_raw;                      // tile keys (bulk copy target, then sorted)
    float *sv = (float *)(smem_raw + S::kCap * 4);
    int *hist = (int *)(smem_raw + S::kCap * 8);            // bucket counts / starts [kNb + 1]
    int *binfo = hist + S::kNb + 8;                         // (bucket start << 16) | keys to rank against
    int *ro = binfo + S::kCap;        // row slot offsets in the tile [nr + 1]
    int *rv = ro + RW;                // products per row
    int *rmn = rv + RW;               // column min / max per row
    int *rmx = rmn + RW;
    int *rss = rmx + RW;              // first sorted position of the row [nr + 1]
    int *rout = rss + RW;             // first merged position of the row
    int *rth = rout + RW;             // first thread of the row [nr + 1] (a row owns ceil(cap / EPT))
    int32_t *tk = (int32_t *)hist;                          // sorted tile (the ranking's output): keys
    float *tv = (float *)(hist + S::kCap);                  //   values
    int32_t *ok = sk;                                       // merged tile (staging of the copy-out)
    float *ov = sv;
    double *lead = (double *)binfo;                         // slice carries: sum before the first head
    int *hhead = (int *)(lead + T);                         //   and whether the slice has a head
    __shared__ uint64_t mbar;
    __shared__ int64_t s_t, s_P;
    __shared__ int sc0[NW + 1], sc1[NW + 1];
    const int tid = threadIdx.x;
    const bool prof_on = a.debug == 2 && tid == 0;
    __shared__ unsigned long long ph[16];
    long long t_last = clock64();
    if (tid < 16) ph[tid] = 0;
    if (tid == 0) {
        mbar_init(&mbar, 1);
        s_t = (int64_t)atomicAdd(a.ticket, 1ull);
    }
    __syncthreads();
    const int64_t NT = *a.ntiles;
    uint32_t phase = 0;
    while (true) {
        const int64_t t = s_t;   // (claimed before the previous barrier)
        if (t >= NT) break;
        const TileDesc d = a.tiles[t];
        if (d.kind == TK_COPY || d.kind == TK_INPLACE) {
            // ---- chunk of merged entries: dense group (scratch) or long row merged in place -----
            const int64_t q0 = (int64_t)d.y * kCopyChunk;
            int64_t Ui, src;
            const int32_t *sc_col;
            const float *sc_val;
            int crow;
            if (d.kind == TK_COPY) {
                Ui = a.lt.g_cnt[d.x];
                src = a.lt.g_off[d.x] + q0;
                sc_col = a.scol;
                sc_val = a.sval;
                crow = d.z;
            } else {
                Ui = a.ccount[d.x];
                src = a.rowoff[d.x] + q0;
                sc_col = a.col;
                sc_val = a.val;
                crow = q0 == 0 ? d.x : -1;
            }
            const int64_t rem = Ui - q0;
            const int U = rem <= 0 ? 0 : (rem < kCopyChunk ? (int)rem : kCopyChunk);
            constexpr int CPT = kCopyChunk / T;
            int32_t ck[CPT];
            float cv[CPT];
#pragma unroll
            for (int j = 0; j < CPT; ++j) {
                const int q = j * T + tid;
                if (q < U) { ck[j] = sc_col[src + q]; cv[j] = sc_val[src + q]; }
            }
            __syncthreads();   // the whole chunk is in registers before its count is published
            if (warp_id() == 0) {
                if (a.debug != 1) lb_publish(a.status, t, U);
                const int64_t P = a.debug == 1 ? src : lb_resolve(a.status, t, U);
                if (lane_id() == 0) {
                    s_P = P;
                    s_t = (int64_t)atomicAdd(a.ticket, 1ull);   // next tile
                }
            }
            __syncthreads();
            const int64_t P = s_P;
            if (tid == 0) {
                if (crow >= 0) a.crowptr[crow] = P;
                if (t == NT - 1) a.crowptr[a.M] = P + U;
            }
#pragma unroll
            for (int j = 0; j < CPT; ++j) {
                const int q = j * T + tid;
                if (q < U) { a.col[P + q] = ck[j]; a.val[P + q] = cv[j]; }
            }
            __syncthreads();   // (s_P is read before the next tile rewrites it)
            if (prof_on) ph[12]++;
            TILE_PH(10);
            continue;
        }
        // ---- rows [r0, r1) of Ĉ, or one column group of a long row (one row, scratch input) ------
        // Row r owns the threads [rth[r], rth[r+1]), ceil(cap_r / EPT) of them: thread t takes the
        // slots ro[r] + EPT (t - rth[r]) + [0, EPT) of its row only (no row tracking per slot).
        const bool grp = d.kind == TK_GROUP;
        int r0, nr, n, lo_in = 0, cnt = 0;
        int64_t S0;
        const int32_t *src_col;
        const float *src_val;
        if (!grp) {
            r0 = d.x;
            nr = d.y - d.x;
            S0 = a.rowoff[r0];
            n = (int)(a.rowoff[d.y] - S0);
            src_col = a.col;
            src_val = a.val;
        } else {   // the group's products [off, off + cnt), loaded from the aligned slot below off
            r0 = d.y;   // (-1: not the row's first group)
            nr = 1;
            const int64_t off = a.lt.g_off[d.x];
            cnt = a.lt.g_cnt[d.x];
            S0 = off & ~(int64_t)3;
            lo_in = (int)(off - S0);
            n = (int)(((off + cnt + 3) & ~(int64_t)3) - S0);
            src_col = a.scol;
            src_val = a.sval;
        }
        {   // row table + thread allotment (one exclusive sum over the rows)
            int nth = 0;
            if (tid < nr) {
                int o0, o1, lv;
                if (!grp) {
                    o0 = (int)(a.rowoff[r0 + tid] - S0);
                    o1 = (int)(a.rowoff[r0 + tid + 1] - S0);
                    lv = (int)a.rowwork[r0 + tid];
                } else {
                    o0 = 0;
                    o1 = n;
                    lv = cnt;
                }
                ro[tid] = o0;
                rv[tid] = lv;
                nth = (o1 - o0 + EPT - 1) / EPT;
            }
            int tot;
            const int th = cta_excl_sum<NW>(nth, sc1, &tot);   // (also the barrier after the previous
            if (tid < nr) rth[tid] = th;                       //  tile's copy-out of sk / sv, rout)
            if (tid == 0) { ro[nr] = n; rth[nr] = tot; }
        }
        if (tid == 0 && n > 0) {
            fence_proxy_async_smem();   // the generic-proxy accesses of sk, sv come first
            mbar_expect_tx(&mbar, (uint32_t)n * 8u);
            bulk_g2s(sk, src_col + S0, (uint32_t)n * 4u, &mbar);
            bulk_g2s(sv, src_val + S0, (uint32_t)n * 4u, &mbar);
        }
        {
            int4 *h4 = reinterpret_cast<int4 *>(hist);
            for (int q = tid; q < (2 * EPT * T) / 4 + 2; q += T) h4[q] = make_int4(0, 0, 0, 0);
            for (int r = tid; r < nr; r += T) { rmn[r] = kKeyPad; rmx[r] = -1; rout[r] = -1; }
        }
        __syncthreads();   // (B1) row table, rth
        TILE_PH(0);
        const int NTH = rth[nr];
        // my row: last r with rth[r] <= tid (rows without slots share the next row's first thread)
        int row = 0;
        if (tid < NTH && nr > 1) {
            int lo = 0, hi = nr;
            while (hi - lo > 1) {
                const int mid = (lo + hi) >> 1;
                if (rth[mid] <= tid) lo = mid; else hi = mid;
            }
            row = lo;
        }
        const bool act = tid < NTH;
        const int k_in_row = tid - rth[row];
        const int ps = ro[row] + EPT * k_in_row;                              // my first slot
        const int rlo = grp ? lo_in : ro[row], rhi = grp ? lo_in + cnt : ro[row + 1];   // my row's slots
        auto load_keys = [&](int32_t (&kk)[EPT]) {
#pragma unroll
            for (int v = 0; v < EPT / 4; ++v) {
                int4 c = make_int4(kKeyPad, kKeyPad, kKeyPad, kKeyPad);
                if (act && ps + 4 * v < n) c = *reinterpret_cast<const int4 *>(sk + ps + 4 * v);
                kk[4 * v] = c.x; kk[4 * v + 1] = c.y; kk[4 * v + 2] = c.z; kk[4 * v + 3] = c.w;
            }
#pragma unroll
            for (int e = 0; e < EPT; ++e)
                if (ps + e < rlo || ps + e >= rhi) kk[e] = kKeyPad;
        };
        if (n > 0) {
            mbar_wait(&mbar, phase);
            phase ^= 1;
        }
        TILE_PH(1);
        {   // per-row column min / max (one pair of shared atomics per thread)
            int32_t key[EPT];
            load_keys(key);
            int lmn = kKeyPad, lmx = -1;
#pragma unroll
            for (int e = 0; e < EPT; ++e)
                if (key[e] != kKeyPad) { lmn = min(lmn, key[e]); lmx = max(lmx, key[e]); }
            if (lmx >= 0) { atomicMin(&rmn[row], lmn); atomicMax(&rmx[row], lmx); }
        }
        __syncthreads();   // (B2)
        TILE_PH(2);
        // ---- histogram: row r's buckets live at [2 EPT rth[r], 2 EPT rth[r+1]) -- 2^floor(log2) of
        //      that many over its column span; the atomic's return value is the key's rank in its
        //      bucket.  bk = bucket | rank << 13 | exact << 26 ------------------------------------------
        int bk[EPT];
        {
            int32_t key[EPT];
            load_keys(key);
            const int base = 2 * EPT * rth[row];
            const int mn = rmn[row];
            const int sh = row_shift(EPT * (rth[row + 1] - rth[row]), mn, rmx[row]);
#pragma unroll
            for (int e = 0; e < EPT; ++e) {
                bk[e] = -1;
                if (key[e] != kKeyPad) {
                    const int b = base + ((key[e] - mn) >> sh);
                    const int rk = atomicAdd(&hist[b], 1);
                    bk[e] = b | (rk << 13) | ((sh == 0) << 26);
                }
            }
        }
        __syncthreads();   // (B3)
        TILE_PH(3);
        // ---- bucket starts: exclusive scan, BPT contiguous buckets per thread ---------------------
        int V;
        {
            const int b0 = tid * BPT;
            int cs = 0;
            if (b0 < 2 * EPT * NTH) {
#pragma unroll
                for (int v = 0; v < BPT / 4; ++v) {
                    const int4 c = *reinterpret_cast<const int4 *>(hist + b0 + 4 * v);
                    cs += c.x + c.y + c.z + c.w;
                }
            }
            int ex = cta_excl_sum<NW>(cs, sc0, &V);   // (B4)
            if (b0 < 2 * EPT * NTH) {
#pragma unroll
                for (int v = 0; v < BPT / 4; ++v) {
                    int4 c = *reinterpret_cast<const int4 *>(hist + b0 + 4 * v);
                    const int x = c.x, y = c.y, z = c.z, w = c.w;
                    c = make_int4(ex, ex + x, ex + x + y, ex + x + y + z);
                    ex += x + y + z + w;
                    *reinterpret_cast<int4 *>(hist + b0 + 4 * v) = c;
                }
            }
            if (tid == 0) hist[2 * EPT * NTH] = V;
        }
        __syncthreads();   // (B5)
        TILE_PH(4);
        if (tid < nr) rss[tid] = hist[2 * EPT * rth[tid]];
        if (tid == 0) rss[nr] = V;
        // ---- scatter by (bucket start + rank); binfo marks the slots that still have to rank -------
        {
            int32_t key[EPT];
            float val[EPT];
            load_keys(key);
#pragma unroll
            for (int v = 0; v < EPT / 4; ++v) {
                float4 f = make_float4(0.f, 0.f, 0.f, 0.f);
                if (act && ps + 4 * v < n) f = *reinterpret_cast<const float4 *>(sv + ps + 4 * v);
                val[4 * v] = f.x; val[4 * v + 1] = f.y; val[4 * v + 2] = f.z; val[4 * v + 3] = f.w;
            }
            __syncthreads();   // (B6: every slot read before the scatter overwrites the tile)
#pragma unroll
            for (int e = 0; e < EPT; ++e) {
                if (bk[e] >= 0) {
                    const int b = bk[e] & 0x1fff;
                    const int bs = hist[b];
                    const int pos = bs + ((bk[e] >> 13) & 0x1fff);
                    sk[pos] = key[e];
                    sv[pos] = val[e];
                    const int c = (bk[e] >> 26) ? 1 : hist[b + 1] - bs;   // exact bucket: in place
                    binfo[pos] = (bs << 16) | c;
                }
            }
        }
        __syncthreads();   // (B7)
        TILE_PH(5);
        // ---- rank inside the multi-key buckets, by slot (a warp covers 32 consecutive slots, so the
        //      lanes of one bucket loop together); every key is copied to its sorted slot in tk / tv --
#pragma unroll
        for (int j = 0; j < EPT; ++j) {
            const int p = j * T + tid;
            if (p < V) {
                const int info = binfo[p];
                const int c = info & 0xffff;
                const int32_t kk = sk[p];
                int dst = p;
                if (c > 1) {
                    const int bs = info >> 16;
                    int rank = 0;
                    if (c <= 4) {   // the common case: straight-line comparisons, no divergent loop
#pragma unroll
                        for (int i = 0; i < 4; ++i) {
                            const int q = bs + i;
                            const int32_t kq = sk[min(q, bs + c - 1)];
                            rank += (i < c) & ((kq < kk) | ((kq == kk) & (q < p)));
                        }
                    } else {
                        for (int q = bs; q < bs + c; ++q) {
                            const int32_t kq = sk[q];
                            rank += (kq < kk) | ((kq == kk) & (q < p));
                        }
                    }
                    dst = bs + rank;
                }
                tk[dst] = kk;
                tv[dst] = sv[p];
            }
        }
        __syncthreads();   // (B8)
        TILE_PH(6);
        // ---- fp64 segmented reduction: my row's sorted positions rss[r] + 9 k + [0, 9) (odd stride:
        //      no bank conflicts; 9 (rth[r+1] - rth[r]) >= the row's products).  A segment ends at a
        //      key change; a slice sums the segments that start in it, its leading positions (the
        //      tail of the previous slice's last segment) go to lead[] for that slice ---------------------
        int U;
        {
            constexpr int E2 = EPT + 1;
            const int rs = rss[row], re = rss[row + 1];
            const int q0 = act ? min(re, rs + E2 * k_in_row) : 0, q1 = act ? min(re, q0 + E2) : 0;
            int32_t kr[E2];
            float vr[E2];
            unsigned hb = 0;
            {
                int32_t prev = q0 > rs ? tk[q0 - 1] : -1;   // (-1: no column; the row start is a head)
#pragma unroll
                for (int j = 0; j < E2; ++j) {
                    const int q = q0 + j;
                    kr[j] = 0;
                    vr[j] = 0.f;
                    if (q < q1) {
                        kr[j] = tk[q];
                        vr[j] = tv[q];
                        hb |= (unsigned)(kr[j] != prev) << j;
                        prev = kr[j];
                    }
                }
            }
            const int nh = __popc(hb);
            double accs = 0.0, lsum = 0.0;
            int32_t lastk = 0;
#pragma unroll
            for (int j = 0; j < E2; ++j) {
                if (q0 + j < q1) {
                    if ((hb >> j) & 1u) {
                        lastk = kr[j];
                        accs = (double)vr[j];
                    } else if (hb & ((1u << j) - 1u)) {
                        accs += (double)vr[j];
                    } else {
                        lsum += (double)vr[j];
                    }
                }
            }
            lead[tid] = lsum;
            hhead[tid] = hb != 0 || q0 >= q1;
            int o = cta_excl_sum<NW>(nh, sc1, &U);   // (B9)
            if (warp_id() == 0 && a.debug != 1) lb_publish(a.status, t, U);
            if (act && k_in_row == 0 && re > rs) rout[row] = o;
            if (nh) {
                // completed segments (all heads but the last), then the last one with its carries
                int oo = o;
                double acc = 0.0;
                int32_t hk = 0;
                bool have = false;
#pragma unroll
                for (int j = 0; j < E2; ++j) {
                    if (q0 + j < q1) {
                        if ((hb >> j) & 1u) {
                            if (have) { ok[oo] = hk; ov[oo] = (float)acc; ++oo; }
                            have = true;
                            hk = kr[j];
                            acc = (double)vr[j];
                        } else if (have) {
                            acc += (double)vr[j];
                        }
                    }
                }
                for (int u = tid + 1; u < NTH; ++u) {   // the last segment continues through slices
                    accs += lead[u];                     // without a head (their lead is all theirs)
                    if (hhead[u]) break;
                }
                ok[oo] = lastk;
                ov[oo] = (float)accs;
            }
        }
        TILE_PH(7);
        if (warp_id() == 0) {
            const int64_t P = a.debug == 1 ? S0 : lb_resolve(a.status, t, U);
            if (lane_id() == 0) {
                s_P = P;
                s_t = (int64_t)atomicAdd(a.ticket, 1ull);   // next tile
            }
        }
        __syncthreads();   // (B10)
        TILE_PH(8);
        // rows without products: the merged position of the next row with products (or U)
        const int64_t P = s_P;
        if (tid < nr && r0 >= 0) {
            int q = tid, ro_ = rout[tid];
            while (ro_ < 0 && ++q < nr) ro_ = rout[q];
            a.crowptr[r0 + tid] = P + (ro_ < 0 ? U : ro_);
        }
        if (tid == 0 && t == NT - 1) a.crowptr[a.M] = P + U;
        for (int q = tid; q < U; q += T) {
            a.col[P + q] = ok[q];
            a.val[P + q] = ov[q];
        }
        if (prof_on) ph[11]++;
        TILE_PH(9);
    }
    if (prof_on)
        for (int k = 0; k < 16; ++k) atomicAdd(a.prof + k, ph[k]);
}

}  // namespace spg
