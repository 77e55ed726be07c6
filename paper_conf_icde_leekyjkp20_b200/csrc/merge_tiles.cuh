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
constexpr int kTileMaxRows = 256;                   // rows of one tile (one thread per row in the row phases)
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
            const int64_t cc = (lane >= done && lane < nin) ? cap : 0;
            const int64_t pre = warp_incl_sum(cc);
            const int64_t first = open >= 0 ? open : w0 + done;   // first row of the tile being grown
            const bool ev = lane >= done && lane < nin &&
                            (lim || acc + pre > kTileCap || (w0 + lane) - first >= kTileMaxRows);
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
                acc = __shfl_sync(kFull, cap, j);
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
};

template <int T, int EPT>
struct TileSmem {
    static constexpr int kCap = T * EPT;
    static constexpr int kNb = 2 * kCap;                  // sum over rows of 2^ceil(log2 Lv) <= 2 * slots
    static constexpr int kHistWords = hidx(kNb) + 4;      // (+ the end-of-tile entry)
    static constexpr int kRowWords = 8 * (kTileMaxRows + 1);
    // layout: keys | vals (bulk copy target, then the sorted tile) | hist (bucket counts / starts; then
    // merged values + slice carries) | binfo (bucket of every scattered slot; then merged keys) | rows
    static constexpr int kBytes = kCap * 8 + kHistWords * 4 + kCap * 4 + kRowWords * 4;
    static_assert(kHistWords * 4 >= kCap * 4 + T * 12, "merged values + carries alias the histogram");
};

template <int T, int EPT>
__global__ void __launch_bounds__(T, 2) k_merge_tiles(TileArgs a) {
    using S = TileSmem<T, EPT>;
    constexpr int NW = T / 32;
    constexpr int RW = kTileMaxRows + 1;
    static_assert(EPT % 4 == 0, "vector loads");
    constexpr int E2M = (S::kCap + T - 1) / T + 1;    // max slice length of the reduction (odd stride)
    extern __shared__ __align__(16) unsigned char smem_raw[];
    int32_t *sk = (int32_t *)smem_raw;                      // tile keys (bulk copy target, then sorted)
    float *sv = (float *)(smem_raw + S::kCap * 4);
    int *hist = (int *)(smem_raw + S::kCap * 8);            // bucket counts / starts
    int *binfo = hist + S::kHistWords;                      // (bucket start << 16) | keys to rank against
    int *ro = binfo + S::kCap;        // row slot offsets in the tile [nr + 1]
    int *rv = ro + RW;                // products per row
    int *rmn = rv + RW;               // column min / max per row
    int *rmx = rmn + RW;
    int *rbb = rmx + RW;              // first bucket of the row [nr + 1]
    int *rsh = rbb + RW;              // bucket shift
    int *rss = rsh + RW;              // first sorted position of the row [nr + 1]
    int *rout = rss + RW;             // first merged position of the row
    int32_t *ok = binfo;              // merged tile (after the ranking): keys
    float *ov = (float *)hist;        //   values
    double *lead = (double *)(hist + S::kCap);             // slice carries: sum before the first head
    int *hhead = (int *)(lead + T);                         //   and whether the slice has a head
    __shared__ uint64_t mbar;
    __shared__ int64_t s_t, s_P;
    __shared__ int sc[NW + 1];
    const int tid = threadIdx.x;
    const Group<NW, 1> g;
    if (tid == 0) mbar_init(&mbar, 1);
    __syncthreads();
    const int64_t NT = *a.ntiles;
    uint32_t phase = 0;
    while (true) {
        if (tid == 0) s_t = (int64_t)atomicAdd(a.ticket, 1ull);
        __syncthreads();
        const int64_t t = s_t;
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
                lb_publish(a.status, t, U);
                const int64_t P = lb_resolve(a.status, t, U);
                if (lane_id() == 0) s_P = P;
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
            continue;
        }
        // ---- rows [r0, r1) of Ĉ, or one column group of a long row (one row, scratch input) ------
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
        if (tid == 0 && n > 0) {
            fence_proxy_async_smem();   // previous tile's reads / writes of sk, sv come first
            mbar_expect_tx(&mbar, (uint32_t)n * 8u);
            bulk_g2s(sk, src_col + S0, (uint32_t)n * 4u, &mbar);
            bulk_g2s(sv, src_val + S0, (uint32_t)n * 4u, &mbar);
        }
        if (!grp) {
            for (int r = tid; r < nr; r += T) {
                ro[r] = (int)(a.rowoff[r0 + r] - S0);
                rv[r] = (int)a.rowwork[r0 + r];
                rmn[r] = kKeyPad;
                rmx[r] = -1;
                rout[r] = -1;
            }
        } else if (tid == 0) {
            ro[0] = 0;
            rv[0] = cnt;
            rmn[0] = kKeyPad;
            rmx[0] = -1;
            rout[0] = -1;
        }
        if (tid == 0) ro[nr] = n;
        {   // zero the histogram (it held the previous tile's merged values, read before the claim)
            int4 *h4 = reinterpret_cast<int4 *>(hist);
            for (int q = tid; q < S::kHistWords / 4; q += T) h4[q] = make_int4(0, 0, 0, 0);
        }
        __syncthreads();
        if (n > 0) {
            mbar_wait(&mbar, phase);
            phase ^= 1;
        }
        // ---- registers: slots [p0, p0 + EPT) of the tile; the row of p0 ---------------------
        const int p0 = tid * EPT;
        int32_t key[EPT];
        float val[EPT];
#pragma unroll
        for (int v = 0; v < EPT / 4; ++v) {
            const int p = p0 + 4 * v;
            int4 c = make_int4(kKeyPad, kKeyPad, kKeyPad, kKeyPad);
            float4 f = make_float4(0.f, 0.f, 0.f, 0.f);
            if (p < n) {
                c = *reinterpret_cast<const int4 *>(sk + p);
                f = *reinterpret_cast<const float4 *>(sv + p);
            }
            key[4 * v] = c.x; key[4 * v + 1] = c.y; key[4 * v + 2] = c.z; key[4 * v + 3] = c.w;
            val[4 * v] = f.x; val[4 * v + 1] = f.y; val[4 * v + 2] = f.z; val[4 * v + 3] = f.w;
        }
        if (grp) {   // slots of the neighbouring groups inside the aligned window are not ours
#pragma unroll
            for (int e = 0; e < EPT; ++e)
                if (p0 + e < lo_in || p0 + e >= lo_in + cnt) key[e] = kKeyPad;
        }
        int row0 = 0;
        if (p0 < n && nr > 1) {
            int lo = 0, hi = nr;
            while (hi - lo > 1) {
                const int mid = (lo + hi) >> 1;
                if (ro[mid] <= p0) lo = mid; else hi = mid;
            }
            row0 = lo;
        }
        {   // per-row column min / max (one pair of shared atomics per row segment of the thread)
            int row = row0, nxt = ro[row0 + 1];
            int cur = -1, lmn = 0, lmx = 0;
#pragma unroll
            for (int e = 0; e < EPT; ++e) {
                const int p = p0 + e;
                if (key[e] != kKeyPad) {
                    while (p >= nxt) { ++row; nxt = ro[row + 1]; }
                    if (row != cur) {
                        if (cur >= 0) { atomicMin(&rmn[cur], lmn); atomicMax(&rmx[cur], lmx); }
                        cur = row;
                        lmn = lmx = key[e];
                    } else {
                        lmn = min(lmn, key[e]);
                        lmx = max(lmx, key[e]);
                    }
                }
            }
            if (cur >= 0) { atomicMin(&rmn[cur], lmn); atomicMax(&rmx[cur], lmx); }
        }
        __syncthreads();
        // ---- per-row bucket parameters; row-major bucket bases -------------------------------
        {
            int nbr = 0;
            if (tid < nr) {
                const int Lv = rv[tid];
                if (Lv > 0) {
                    const uint32_t span = (uint32_t)(rmx[tid] - rmn[tid]);
                    const int lognb = nextpow2_log(Lv);
                    const int bits = span ? 32 - __clz(span) : 0;
                    const int sh = max(0, bits - lognb);
                    rsh[tid] = sh;
                    nbr = (int)(span >> sh) + 1;
                }
            }
            int NB;
            const int bb = g.excl_sum1(nbr, sc, &NB);
            if (tid < nr) rbb[tid] = bb;
            if (tid == 0) rbb[nr] = NB;
        }
        __syncthreads();
        // ---- histogram: the returned count is the key's rank inside its bucket ---------------
        int bk[EPT], rk[EPT];   // bucket (bit 30: exact bucket, all keys equal; -1: no key), rank
        {
            int row = row0, nxt = ro[row0 + 1];
            int base = rbb[row], mn = rmn[row], sh = rsh[row];
#pragma unroll
            for (int e = 0; e < EPT; ++e) {
                const int p = p0 + e;
                bk[e] = -1;
                rk[e] = 0;
                if (key[e] != kKeyPad) {
                    if (p >= nxt) {
                        do { ++row; nxt = ro[row + 1]; } while (p >= nxt);
                        base = rbb[row];
                        mn = rmn[row];
                        sh = rsh[row];
                    }
                    const int b = base + ((key[e] - mn) >> sh);
                    rk[e] = atomicAdd(&hist[hidx(b)], 1);
                    bk[e] = b | (sh == 0 ? (1 << 30) : 0);
                }
            }
        }
        __syncthreads();
        // ---- bucket starts: exclusive scan (each thread a contiguous range of buckets) -------
        int V;
        {
            const int NB = rbb[nr];
            const int bpt = (NB + T - 1) / T;
            const int b0 = min(NB, tid * bpt), b1 = min(NB, b0 + bpt);
            int cnt = 0;
            for (int b = b0; b < b1; ++b) cnt += hist[hidx(b)];
            int ex = g.excl_sum1(cnt, sc, &V);
            __syncthreads();   // (excl_sum1: the warp totals are read before the next write of sc)
            for (int b = b0; b < b1; ++b) {
                const int c = hist[hidx(b)];
                hist[hidx(b)] = ex;
                ex += c;
            }
            if (tid == 0) hist[hidx(NB)] = V;
        }
        __syncthreads();
        if (tid < nr) rss[tid] = hist[hidx(rbb[tid])];
        if (tid == 0) rss[nr] = V;   // (nr may equal T)
        // ---- scatter by (bucket start + rank); binfo marks the slots that still have to rank -------
#pragma unroll
        for (int e = 0; e < EPT; ++e) {
            if (bk[e] >= 0) {
                const int b = bk[e] & ((1 << 30) - 1);
                const int bs = hist[hidx(b)];
                const int pos = bs + rk[e];
                sk[pos] = key[e];
                sv[pos] = val[e];
                const int c = (bk[e] >> 30) ? 1 : hist[hidx(b + 1)] - bs;   // exact bucket: in place
                binfo[pos] = (bs << 16) | c;
            }
        }
        __syncthreads();
        // ---- rank inside the multi-key buckets, by slot: a warp covers 32 consecutive slots, so
        //      the lanes of one bucket loop together (broadcast reads of the bucket's keys) ----------
        int np[EPT];
        int32_t mk[EPT];
        float mv[EPT];
#pragma unroll
        for (int j = 0; j < EPT; ++j) {
            const int p = j * T + tid;
            np[j] = -1;
            if (p < V) {
                const int info = binfo[p];
                const int c = info & 0xffff;
                if (c > 1) {
                    const int bs = info >> 16;
                    const int32_t kk = sk[p];
                    int rank = 0;
                    for (int q = bs; q < bs + c; ++q) {
                        const int32_t kq = sk[q];
                        rank += (kq < kk) | ((kq == kk) & (q < p));
                    }
                    np[j] = bs + rank;
                    mk[j] = kk;
                    mv[j] = sv[p];
                }
            }
        }
        __syncthreads();
#pragma unroll
        for (int j = 0; j < EPT; ++j)
            if (np[j] >= 0) { sk[np[j]] = mk[j]; sv[np[j]] = mv[j]; }
        __syncthreads();
        // ---- fp64 segmented reduction over contiguous slices (odd stride: no bank conflicts).
        //      A segment ends at a key change or a row start; a slice sums the segments that start
        //      in it, and its leading positions (the tail of the previous slice's last segment) go
        //      to lead[] for that slice to add ----------------------------------------------------------
        int U;
        {
            const int E2 = ((V + T - 1) / T) | 1;
            const int q0 = min(V, tid * E2), q1 = min(V, q0 + E2);
            int row = 0;
            if (q0 < q1 && nr > 1) {
                int lo = 0, hi = nr;   // last row with rss <= q0 (empty rows share the next row's start)
                while (hi - lo > 1) {
                    const int mid = (lo + hi) >> 1;
                    if (rss[mid] <= q0) lo = mid; else hi = mid;
                }
                row = lo;
            }
            int32_t kr[E2M];
            float vr[E2M];
            unsigned hb = 0, rsb = 0;   // head bits and row-start bits of the slice
            {
                int st = rss[row], nx = rss[row + 1], rw = row;
                int32_t prev = q0 > 0 ? sk[q0 - 1] : -1;
#pragma unroll
                for (int j = 0; j < E2M; ++j) {
                    const int q = q0 + j;
                    kr[j] = kKeyPad;
                    vr[j] = 0.f;
                    if (q < q1) {
                        kr[j] = sk[q];
                        vr[j] = sv[q];
                        while (q >= nx) { ++rw; st = nx; nx = rss[rw + 1]; }
                        const bool rs = q == st;
                        hb |= (unsigned)(rs | (kr[j] != prev)) << j;
                        rsb |= (unsigned)rs << j;
                        prev = kr[j];
                    }
                }
            }
            const int nh = __popc(hb);
            int o = g.excl_sum1(nh, sc, &U);
            if (warp_id() == 0) lb_publish(a.status, t, U);
            // slice partial sums: lead = positions before the first head; one sum per head
            double accs = 0.0;
            int last = -1;
            {
                double lsum = 0.0;
#pragma unroll
                for (int j = 0; j < E2M; ++j) {
                    if (q0 + j < q1) {
                        if ((hb >> j) & 1u) {
                            if (last >= 0) {   // close the previous segment of the slice
                                ok[o] = kr[last];
                                ov[o] = (float)accs;
                                ++o;
                            }
                            last = j;
                            accs = (double)vr[j];
                        } else if (last >= 0) {
                            accs += (double)vr[j];
                        } else {
                            lsum += (double)vr[j];
                        }
                    }
                }
                lead[tid] = lsum;
                hhead[tid] = hb != 0 || q0 >= q1;
            }
            __syncthreads();
            if (last >= 0) {   // the slice's last segment may continue through the next slices
                for (int u = tid + 1; u < T; ++u) {
                    accs += lead[u];
                    if (hhead[u]) break;
                }
                ok[o] = kr[last];
                ov[o] = (float)accs;
            }
            // merged index of every row start (the row's first head)
            if (rsb) {
                const int o0 = o - (last >= 0 ? nh - 1 : 0);   // merged index of the slice's first head
                int rw = row;
                for (unsigned m = rsb; m; m &= m - 1) {
                    const int j = __ffs(m) - 1;
                    while (rss[rw + 1] <= q0 + j) ++rw;   // the (non-empty) row starting at q0 + j
                    rout[rw] = o0 + __popc(hb & ((1u << j) - 1u));
                }
            }
        }
        __syncthreads();
        if (warp_id() == 0) {
            const int64_t P = lb_resolve(a.status, t, U);
            if (lane_id() == 0) s_P = P;
        }
        // rows without products: the merged position of the next row with products (or U)
        if (tid < nr && rout[tid] < 0) {
            int q = tid + 1;
            while (q < nr && rout[q] < 0) ++q;
            rout[tid] = q < nr ? rout[q] : U;
        }
        __syncthreads();
        const int64_t P = s_P;
        if (tid < nr && r0 >= 0) a.crowptr[r0 + tid] = P + rout[tid];
        if (tid == 0 && t == NT - 1) a.crowptr[a.M] = P + U;
        for (int q = tid; q < U; q += T) {
            a.col[P + q] = ok[q];
            a.val[P + q] = ov[q];
        }
    }
}

}  // namespace spg
