// Stage (4) merge, B-Limited rows: column-range partition into groups that the merge-tile kernel
// sorts like short rows (§IV-D L463-L477 L: long rows get blocks with extra shared memory,
// which limits the resident blocks per SM -- "B-Limiting").
//
// B200 design ("long rows"): a row whose padded Ĉ bucket exceeds one merge tile is
// cut by column ranges into *groups* of at most kGroupCap products.  One partition CTA per row
// (persistent grid of limit_ctas_per_sm CTAs per SM, longest rows first; 96 KB of shared memory
// each, so at most two are resident per SM):
//   1. histogram of the row's columns over NB1 equal-width bins (bin width 2^sh1 <= kDenseWidth);
//   2. one warp packs consecutive bins greedily into groups of <= kGroupCap products; a bin
//      holding more than kGroupCap products (hub columns repeated across many runs) becomes a
//      *dense group* of its own;
//   3. every product is scattered into its group's range of the scratch buffer (shared-memory
//      cursor per group), so each group is a contiguous, unordered list of one column range.
// Dense groups are merged by k_long_dense (fp64 accumulator over the bin's <= kDenseWidth columns,
// warp-aggregated shared atomics) in place in the scratch; the merge-tile kernel then sorts +
// reduces every other group as one tile and moves the dense groups' merged entries, all in row
// order, straight to C.
#pragma once
#include "merge_tiles.cuh"

namespace spg {

constexpr int kPartT = 512;                  // threads of a partition CTA
constexpr int kPartBins = 8192;              // max level-1 bins of a row
constexpr int kPartGroups = 4096;            // max groups of a row
constexpr int kDenseWidth = 16384;           // max columns of a bin (one fp64 window of a dense group)
constexpr int kDenseT = 1024;
constexpr int64_t kLongMaxL = 4000000;       // longer rows (or wider spans) take the legacy long-row path
constexpr int kPartSmem = (kPartBins + 4 * kPartGroups) * 4;
constexpr int kDenseSmem = kDenseWidth * 8 + (kDenseWidth / 32) * 4;
static_assert(kGroupCap + 8 <= kTileCap, "a group tile loads up to 3 + 3 extra aligned slots");

enum : int8_t { GK_SORT = 0, GK_DENSE = 1, GK_MERGED = 2 };

// group-table bound of a row with Lv products: consecutive normal groups hold > kGroupCap products
// together and a dense group alone does, so G <= 4 * ceil(Lv / kGroupCap) + 4
__host__ __device__ __forceinline__ int64_t long_group_bound(int64_t Lv) {
    return 4 * ((Lv + kGroupCap - 1) / kGroupCap) + 4;
}

// per limited row q (list order): scratch slots and group-table slots (scanned by the host)
__global__ void k_long_sizes(const int32_t *__restrict__ rows, int64_t nrows, const int64_t *__restrict__ rowwork,
                             int64_t *__restrict__ xs, int64_t *__restrict__ ys) {
    for (int64_t q = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; q < nrows; q += (int64_t)gridDim.x * blockDim.x) {
        const int64_t Lv = rowwork[rows[q]];
        xs[q] = pad_run(Lv);
        ys[q] = long_group_bound(Lv);
    }
}

struct LongArgs {
    const int32_t *rows;             // limited rows, longest first
    int64_t nrows;
    const int64_t *rowoff, *rowwork;
    const int32_t *rowmn, *rowmx;    // exact column range of every long row (spgemm_plan, R12)
    const int32_t *col;              // Ĉ
    const float *val;
    const int64_t *xoff, *yoff;      // scratch / group-table offset of list entry q
    int32_t *scol;                   // scratch
    float *sval;
    int64_t *g_off;                  // group table: scratch offset, products (merged count after
    int32_t *g_cnt;                  //   k_long_dense), first column (dense groups), kind
    int32_t *g_lo;
    int8_t *g_kind;
    int32_t *g_num;                  // groups of list entry q
    int64_t *dense_list;             // global indices of the dense groups
    unsigned long long *dense_count;
    unsigned long long *counter;     // row claim ticket
};

__device__ __forceinline__ int span_bits(uint32_t span) { return span ? 32 - __clz(span) : 0; }

__global__ void __launch_bounds__(kPartT) k_long_partition(LongArgs a) {
    extern __shared__ __align__(16) unsigned char smem_raw[];
    int *hist = (int *)smem_raw;                 // bin counts, then the bin -> group map
    int *gcnt = hist + kPartBins;                // products per group
    int *goff = gcnt + kPartGroups;              // group offset inside the row's scratch range
    int *gcur = goff + kPartGroups;              // scatter cursors
    int *glo = gcur + kPartGroups;               // first bin of a group
    __shared__ int64_t s_q;
    __shared__ int s_G;
    const int tid = threadIdx.x;
    while (true) {
        if (tid == 0) s_q = (int64_t)atomicAdd(a.counter, 1ull);
        __syncthreads();
        const int64_t q = s_q;
        if (q >= a.nrows) break;
        const int i = a.rows[q];
        const int64_t S = a.rowoff[i];
        const int64_t cap = a.rowoff[i + 1] - S;
        const int64_t Lv = a.rowwork[i];
        int mn = a.rowmn[i], mx = a.rowmx[i];
        const int4 *k4 = reinterpret_cast<const int4 *>(a.col + S);
        if (mn > mx) {   // range not recorded by the plan (rows of <= 256 slots, Limited by the β threshold)
            int lmn = kKeyPad, lmx = -1;
            for (int64_t v = tid; v < cap / 4; v += kPartT) {
                const int4 c = __ldg(k4 + v);
                const int32_t kk[4] = {c.x, c.y, c.z, c.w};
#pragma unroll
                for (int e = 0; e < 4; ++e)
                    if (kk[e] != kKeyPad) { lmn = min(lmn, kk[e]); lmx = max(lmx, kk[e]); }
            }
            if (tid == 0) { gcnt[0] = kKeyPad; gcnt[1] = -1; }
            __syncthreads();
            lmn = warp_min(lmn);
            lmx = warp_max(lmx);
            if (lane_id() == 0) { atomicMin(&gcnt[0], lmn); atomicMax(&gcnt[1], lmx); }
            __syncthreads();
            mn = gcnt[0];
            mx = gcnt[1];
            __syncthreads();
        }
        const uint32_t span = (uint32_t)(mx - mn);
        const int bits = span_bits(span);
        // NB1 = 2^lb bins: about 8 products per bin, and bins at most kDenseWidth columns wide
        const int64_t per8 = Lv / 8 + 1;
        int lb = max(8, nextpow2_log((int)(per8 < kPartBins ? per8 : kPartBins)));
        lb = max(lb, bits - 14);
        const int sh1 = max(0, bits - lb);
        const int nbins = (int)(span >> sh1) + 1;
        for (int b = tid; b < nbins; b += kPartT) hist[b] = 0;
        __syncthreads();
        // ---- 1. column histogram -----------------------------------------------------------
        for (int64_t v = tid; v < cap / 4; v += kPartT) {
            const int4 c = __ldg(k4 + v);
            if (c.x != kKeyPad) atomicAdd(&hist[(c.x - mn) >> sh1], 1);
            if (c.y != kKeyPad) atomicAdd(&hist[(c.y - mn) >> sh1], 1);
            if (c.z != kKeyPad) atomicAdd(&hist[(c.z - mn) >> sh1], 1);
            if (c.w != kKeyPad) atomicAdd(&hist[(c.w - mn) >> sh1], 1);
        }
        __syncthreads();
        // ---- 2. greedy grouping of consecutive bins (one warp) -------------------------------
        if (tid < 32) {
            const int lane = tid;
            int g = 0, acc = 0;
            bool open = false;
            for (int base = 0; base < nbins; base += 32) {
                const int b = base + lane;
                const int c = b < nbins ? hist[b] : 0;
                int done = 0;
                while (done < 32) {
                    const int cc = lane >= done ? c : 0;
                    const int pre = warp_incl_sum(cc);
                    const bool ev = lane >= done && (c > kGroupCap || acc + pre > kGroupCap);
                    const unsigned m = __ballot_sync(kFull, ev);
                    const int j = m ? __ffs(m) - 1 : 32;
                    if (lane >= done && lane < j && b < nbins) hist[b] = g;   // joins the open group
                    const int add = j > done ? __shfl_sync(kFull, pre, j - 1) : 0;
                    acc += add;
                    open = open || add > 0;
                    if (j == 32) break;
                    const int cj = __shfl_sync(kFull, c, j);
                    if (cj > kGroupCap) {          // dense group: this bin alone
                        if (open) {
                            if (lane == 0) gcnt[g] = acc;
                            ++g;
                        }
                        if (lane == 0) { gcnt[g] = -cj; glo[g] = base + j; }   // (negative: dense)
                        if (lane == j) hist[b] = g;
                        ++g;
                        acc = 0;
                        open = false;
                    } else {                        // the open group is full: bin j starts the next
                        if (lane == 0) gcnt[g] = acc;
                        ++g;
                        acc = cj;
                        open = true;
                        if (lane == j) hist[b] = g;
                    }
                    done = j + 1;
                }
            }
            if (open) {
                if (lane == 0) gcnt[g] = acc;
                ++g;
            }
            // group offsets inside the row's scratch range (exclusive prefix of |count|)
            int run = 0;
            for (int g0 = 0; g0 < g; g0 += 32) {
                const int c = g0 + lane < g ? abs(gcnt[g0 + lane]) : 0;
                const int inc = warp_incl_sum(c);
                if (g0 + lane < g) { goff[g0 + lane] = run + inc - c; gcur[g0 + lane] = 0; }
                run += __shfl_sync(kFull, inc, 31);
            }
            if (lane == 0) s_G = g;
        }
        __syncthreads();
        const int G = s_G;
        const int64_t X = a.xoff[q];
        // ---- 3. scatter into the groups --------------------------------------------------------
        const float4 *v4 = reinterpret_cast<const float4 *>(a.val + S);
        for (int64_t v = tid; v < cap / 4; v += kPartT) {
            const int4 c = __ldg(k4 + v);
            const float4 f = __ldg(v4 + v);
            const int32_t kk[4] = {c.x, c.y, c.z, c.w};
            const float vv[4] = {f.x, f.y, f.z, f.w};
#pragma unroll
            for (int e = 0; e < 4; ++e) {
                if (kk[e] != kKeyPad) {
                    const int gg = hist[(kk[e] - mn) >> sh1];
                    const int64_t pos = X + goff[gg] + atomicAdd(&gcur[gg], 1);
                    a.scol[pos] = kk[e];
                    a.sval[pos] = vv[e];
                }
            }
        }
        // ---- group table ------------------------------------------------------------------------
        const int64_t Y = a.yoff[q];
        for (int g = tid; g < G; g += kPartT) {
            const int c = gcnt[g];
            a.g_off[Y + g] = X + goff[g];
            a.g_cnt[Y + g] = abs(c);
            if (c < 0) {
                a.g_kind[Y + g] = GK_DENSE;
                a.g_lo[Y + g] = mn + (glo[g] << sh1);
                a.dense_list[atomicAdd(a.dense_count, 1ull)] = Y + g;
            } else {
                a.g_kind[Y + g] = GK_SORT;
            }
        }
        if (tid == 0) a.g_num[q] = G;
        __syncthreads();
    }
}

// Dense groups: every product of one bin of <= kDenseWidth columns, summed in an fp64 shared
// accumulator (a warp whose 32 products share one column adds once), emitted in column order in
// place at the head of the group's scratch range; g_cnt becomes the merged count.
__global__ void __launch_bounds__(kDenseT, 1) k_long_dense(const int64_t *__restrict__ list,
                                                           const unsigned long long *__restrict__ count,
                                                           const int64_t *__restrict__ g_off,
                                                           int32_t *__restrict__ g_cnt, const int32_t *__restrict__ g_lo,
                                                           int8_t *__restrict__ g_kind, int32_t *__restrict__ scol,
                                                           float *__restrict__ sval) {
    extern __shared__ __align__(16) unsigned char smem_raw[];
    double *acc = (double *)smem_raw;
    uint32_t *bits = (uint32_t *)(smem_raw + kDenseWidth * 8);
    __shared__ int sc[kDenseT / 32 + 1];
    const int tid = threadIdx.x;
    const Group<kDenseT / 32, 1> grp;
    const int64_t n = (int64_t)*count;
    for (int64_t d = blockIdx.x; d < n; d += gridDim.x) {
        const int64_t gi = list[d];
        const int64_t off = g_off[gi];
        const int cnt = g_cnt[gi];
        const int lo = g_lo[gi];
        for (int c = tid; c < kDenseWidth; c += kDenseT) acc[c] = 0.0;
        for (int w = tid; w < kDenseWidth / 32; w += kDenseT) bits[w] = 0;
        __syncthreads();
        for (int p0 = 0; p0 < cnt; p0 += kDenseT) {   // (warp-uniform trip count)
            const int p = p0 + tid;
            const bool ok = p < cnt;
            const int c = ok ? scol[off + p] - lo : -1;
            const double v = ok ? (double)sval[off + p] : 0.0;
            const int c0 = __shfl_sync(kFull, c, 0);
            if (__all_sync(kFull, c == c0 && ok)) {   // one column for the whole warp (hub duplicates)
                const double s = warp_sum(v);
                if (lane_id() == 0) {
                    atomicAdd(&acc[c0], s);
                    atomicOr(&bits[c0 >> 5], 1u << (c0 & 31));
                }
            } else if (ok) {
                atomicAdd(&acc[c], v);
                atomicOr(&bits[c >> 5], 1u << (c & 31));
            }
        }
        __syncthreads();
        // emit in column order: thread t owns the columns [16 t, 16 t + 16)
        constexpr int CPT = kDenseWidth / kDenseT;
        static_assert(CPT == 16, "one half bitmap word per thread");
        const uint32_t word = bits[tid >> 1] >> ((tid & 1) * 16) & 0xffffu;
        int U;
        int o = grp.excl_sum(__popc(word), sc, &U);
        for (uint32_t w = word; w; w &= w - 1) {
            const int c = tid * CPT + __ffs(w) - 1;
            scol[off + o] = lo + c;
            sval[off + o] = (float)acc[c];
            ++o;
        }
        if (tid == 0) {
            g_cnt[gi] = U;
            g_kind[gi] = GK_MERGED;
        }
        __syncthreads();
    }
}

}  // namespace spg
