// Stage (4) merge of the short rows, fused with the CSR compaction.
//
// PAPER.md §IV-D L452-L477 L: "elements with the same indices are merged into unique elements";
// BASELINE.json north_star: "a row-bucketed sort plus segmented reduce into CSR".
//
// B200 design ("units"): consecutive short rows (padded bucket <= kUnitRowMax
// slots) are grouped into *units* -- all rows whose Ĉ bucket starts in the same kUnitWindow-slot
// window of the padded offsets, so a unit holds < kUnitCap slots -- and every long row
// (B-Limited or > kUnitRowMax slots; merged beforehand by merge.cuh into the side buffer) is a
// unit of its own.  One persistent kernel claims units in row order (atomic ticket) and per unit:
//   1. loads the unit's slots (16-byte vectors, contiguous per thread) into registers; per-row
//      column min / max by shared atomics;
//   2. per row nb = span-clipped 2^ceil(log2 L) buckets, (col - min) >> sh; the unit's buckets are
//      row-major, so one histogram (shared atomics, rank = returned count) + one scan orders the
//      whole unit by (row, column bucket);
//   3. singleton buckets land directly in their sorted slot; the rest rank against the keys of
//      their bucket (equal keys by scatter position);
//   4. fp64 segmented reduction (a segment ends at a key change or a row start) into a compact
//      staging copy of the merged unit;
//   5. decoupled look-back over the units' merged counts gives the unit's output offset P;
//      it writes C's row pointers and its merged rows at [P, P + U) -- in place in the Ĉ arrays,
//      which is safe because P <= the unit's first slot, and every earlier unit has loaded its
//      input before publishing the count this unit waited for.
// A long-row unit publishes ccount (known) at once and copies its merged row from the side
// buffer.  A unit with a bucket of > kBucketMax keys (clustered columns) falls back to a per-row
// natural merge sort in shared memory.  No separate compaction pass exists: the merge reads Ĉ
// once and writes C once.
#pragma once
#include "merge.cuh"

namespace spg {

constexpr int kMergeFused = 4;                       // options.reserved[0] selecting this merge
constexpr int kUnitCap = 4096;                       // slots of one unit (shared-memory capacity)
constexpr int kUnitThreads = 256;                    // threads per unit CTA (also max rows per unit)
constexpr int kUnitWindow = kUnitCap - kUnitRowMax;  // window of unit starts on the Ĉ offsets
constexpr int kUnitNbMax = 2 * kUnitCap;             // sum over rows of nextpow2(L) <= 2 * slots

__host__ __device__ __forceinline__ bool unit_long_row(int64_t cap, int8_t cls) {
    return cap > kUnitRowMax || cls == RC_LIMITED;
}

// unit starts: row 0, every rows_max-th row, long rows, rows after a long row, window changes
__global__ void k_unit_flags(const int64_t *__restrict__ rowoff, const int8_t *__restrict__ rcls, int64_t M,
                             int rows_max, int32_t *__restrict__ flag, int64_t *__restrict__ longcap) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < M; i += (int64_t)gridDim.x * blockDim.x) {
        const int64_t o = rowoff[i], cap = rowoff[i + 1] - o;
        const bool lg = unit_long_row(cap, rcls[i]);
        bool f = i == 0 || (i % rows_max) == 0 || lg;
        if (!f) {
            const int64_t op = rowoff[i - 1];
            f = unit_long_row(o - op, rcls[i - 1]) || (o / kUnitWindow) != (op / kUnitWindow);
        }
        flag[i] = f;
        longcap[i] = lg ? cap : 0;
    }
}

__global__ void k_unit_rows(const int32_t *__restrict__ flag, const int64_t *__restrict__ uoff, int64_t M,
                            int32_t *__restrict__ unit_row, int64_t *__restrict__ nunits) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < M; i += (int64_t)gridDim.x * blockDim.x) {
        if (flag[i]) unit_row[uoff[i]] = (int32_t)i;
        if (i == 0) {
            unit_row[uoff[M]] = (int32_t)M;
            *nunits = uoff[M];
        }
    }
}

struct UnitArgs {
    const int32_t *unit_row;       // [nunits + 1] first row of every unit
    const int64_t *nunits;         // device scalar
    const int64_t *rowoff;         // padded Ĉ offsets [M + 1]
    const int64_t *rowwork;        // products per row
    const int8_t *rcls;
    int32_t *chat_col;             // in: Ĉ; out: C's columns at [0, nnz(C))
    float *chat_val;
    const int32_t *side_col;       // merged long rows
    const float *side_val;
    const int64_t *side_off;
    const int64_t *ccount;         // merged length of the long rows
    int64_t *crowptr;              // out: C row pointers [M + 1]
    int64_t M;
    unsigned long long *status;    // look-back words [nunits], zeroed
    unsigned long long *ticket;    // zeroed
    unsigned long long *n_fallback;
    int debug;                     // options.reserved[1] (tuning only): 1 = no look-back (wrong C),
                                   // 2 = per-phase clock64 totals of thread 0 into prof[0..16)
    unsigned long long *prof;
};
#define UNIT_PH(k)                                                   \
    do {                                                             \
        if (prof_on) {                                               \
            const long long _t = clock64();                          \
            ph[k] += (unsigned long long)(_t - t_last);              \
            t_last = _t;                                             \
        }                                                            \
    } while (0)

template <int T>
struct UnitSmem {
    static constexpr int kHist = hidx(kUnitNbMax) + 4;
    static constexpr int kBounds = (kUnitCap + 1) + (kUnitCap / 2 + 2);   // natural merge sort fallback
    static constexpr int kHistWords = kHist > kBounds ? kHist : kBounds;
    static constexpr int kRowArrays = 8;
    static constexpr int kBytes = kUnitCap * 16 + kHistWords * 4 + kRowArrays * (T + 1) * 4;
};

template <int T>
__global__ void __launch_bounds__(T, 2) k_merge_units(UnitArgs a) {
    constexpr int EPT = kUnitCap / T;
    constexpr int NW = T / 32;
    using S = UnitSmem<T>;
    static_assert(EPT % 4 == 0, "vector loads");
    extern __shared__ __align__(16) unsigned char smem_raw[];
    int32_t *k0 = (int32_t *)smem_raw;
    float *v0 = (float *)(smem_raw + kUnitCap * 4);
    int32_t *k1 = (int32_t *)(smem_raw + kUnitCap * 8);
    float *v1 = (float *)(smem_raw + kUnitCap * 12);
    int *hist = (int *)(smem_raw + kUnitCap * 16);
    int *ro = hist + S::kHistWords;   // row slot offsets inside the unit [nr + 1]
    int *rv = ro + (T + 1);           // products per row
    int *rbb = rv + (T + 1);          // first bucket of the row [nr + 1]
    int *rsh = rbb + (T + 1);         // bucket shift
    int *rmn = rsh + (T + 1);         // column min / max
    int *rmx = rmn + (T + 1);
    int *rss = rmx + (T + 1);         // first sorted position of the row [nr + 1]
    int *rout = rss + (T + 1);        // first merged position of the row
    __shared__ int sc[NW + 1];
    __shared__ int64_t s_u, s_P;
    const Group<NW, 1> g;
    const int tid = threadIdx.x;
    const int64_t NU = *a.nunits;
    const bool prof_on = a.debug == 2 && tid == 0;
    unsigned long long ph[16] = {};
    long long t_last = clock64();
    while (true) {
        if (tid == 0) s_u = (int64_t)atomicAdd(a.ticket, 1ull);
        __syncthreads();
        UNIT_PH(0);
        const int64_t u = s_u;
        if (u >= NU) break;
        const int r0 = a.unit_row[u], r1 = a.unit_row[u + 1];
        const int nr = r1 - r0;
        const int64_t S0 = a.rowoff[r0];
        const int64_t n64 = a.rowoff[r1] - S0;
        UNIT_PH(1);
        if (nr == 1 && unit_long_row(n64, a.rcls[r0])) {
            if (prof_on) ph[14]++;
            // ---- long row: merged already (side buffer); k_copy_long moves it to [P, P + U)
            const int64_t U = a.ccount[r0];
            if (warp_id() == 0) {
                lb_publish(a.status, u, U);
                const int64_t P = a.debug == 1 ? S0 : lb_resolve(a.status, u, U);
                if (lane_id() == 0) {
                    a.crowptr[r0] = P;
                    if (r1 == a.M) a.crowptr[a.M] = P + U;
                }
            }
            UNIT_PH(13);
            continue;
        }
        if (prof_on) ph[15]++;
        const int n = (int)n64;
        // ---- A: row table
        for (int r = tid; r < nr; r += T) {
            ro[r] = (int)(a.rowoff[r0 + r] - S0);
            rv[r] = (int)a.rowwork[r0 + r];
            rmn[r] = 0x7fffffff;
            rmx[r] = (int)0x80000000;
        }
        if (tid == 0) ro[nr] = n;
        __syncthreads();
        UNIT_PH(2);
        // ---- B: contiguous slots of this thread -> registers; row of every slot; row min / max
        const int pb = tid * EPT;
        int32_t key[EPT];
        float val[EPT];
        int rowe[EPT];
#pragma unroll
        for (int v = 0; v < EPT / 4; ++v) {
            const int p = pb + 4 * v;
            int4 c = make_int4(kKeyPad, kKeyPad, kKeyPad, kKeyPad);
            float4 f = make_float4(0.f, 0.f, 0.f, 0.f);
            if (p < n) {
                c = *reinterpret_cast<const int4 *>(a.chat_col + S0 + p);
                f = *reinterpret_cast<const float4 *>(a.chat_val + S0 + p);
            }
            key[4 * v] = c.x; key[4 * v + 1] = c.y; key[4 * v + 2] = c.z; key[4 * v + 3] = c.w;
            val[4 * v] = f.x; val[4 * v + 1] = f.y; val[4 * v + 2] = f.z; val[4 * v + 3] = f.w;
        }
        {
            int row = 0;
            if (pb < n) {
                int lo = 0, hi = nr;
                while (hi - lo > 1) {
                    const int mid = (lo + hi) >> 1;
                    if (ro[mid] <= pb) lo = mid; else hi = mid;
                }
                row = lo;
            }
            int nxt = ro[row + 1];
            int cur = -1, lmn = 0, lmx = 0;
#pragma unroll
            for (int e = 0; e < EPT; ++e) {
                const int p = pb + e;
                rowe[e] = -1;
                if (p < n) {
                    while (p >= nxt) { ++row; nxt = ro[row + 1]; }
                    if (key[e] != kKeyPad) {
                        rowe[e] = row;
                        if (row != cur) {
                            if (cur >= 0) { atomicMin(&rmn[cur], lmn); atomicMax(&rmx[cur], lmx); }
                            cur = row;
                            lmn = key[e];
                            lmx = key[e];
                        } else {
                            lmn = min(lmn, key[e]);
                            lmx = max(lmx, key[e]);
                        }
                    }
                }
            }
            if (cur >= 0) { atomicMin(&rmn[cur], lmn); atomicMax(&rmx[cur], lmx); }
        }
        __syncthreads();
        UNIT_PH(3);
        // ---- C: per-row bucket parameters, row-major bucket bases
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
        const int bb = g.excl_sum(nbr, sc, &NB);
        if (tid < nr) rbb[tid] = bb;
        if (tid == 0) rbb[nr] = NB;
        for (int b = tid; b <= NB; b += T) hist[hidx(b)] = 0;
        __syncthreads();
        UNIT_PH(4);
        // ---- D: histogram; the atomic's return value is the key's rank inside its bucket
        int bk[EPT], rk[EPT];
#pragma unroll
        for (int e = 0; e < EPT; ++e) {
            bk[e] = -1;
            rk[e] = 0;
            if (rowe[e] >= 0) {
                const int r = rowe[e];
                bk[e] = rbb[r] + ((key[e] - rmn[r]) >> rsh[r]);
                rk[e] = atomicAdd(&hist[hidx(bk[e])], 1);
            }
        }
        __syncthreads();
        UNIT_PH(5);
        // ---- E: exclusive scan of the bucket counts (contiguous bucket ranges per thread)
        int V;
        int big;
        {
            const int bpt = (NB + T - 1) / T;
            const int b0 = min(NB, tid * bpt), b1 = min(NB, b0 + bpt);
            int cnt = 0, mxc = 0;
            for (int b = b0; b < b1; ++b) {
                const int c = hist[hidx(b)];
                cnt += c;
                mxc = max(mxc, c);
            }
            int ex = g.excl_sum(cnt, sc, &V);
            big = g.reduce_max(mxc, sc);
            for (int b = b0; b < b1; ++b) {
                const int c = hist[hidx(b)];
                hist[hidx(b)] = ex;
                ex += c;
            }
            if (tid == 0) hist[hidx(NB)] = V;
        }
        __syncthreads();
        UNIT_PH(6);
        int U;
        if (big <= kBucketMax) {
            if (tid <= nr) rss[tid] = hist[hidx(rbb[tid])];
            // ---- F: scatter; singleton buckets are final
#pragma unroll
            for (int e = 0; e < EPT; ++e) {
                if (bk[e] >= 0) {
                    const int bs = hist[hidx(bk[e])], be = hist[hidx(bk[e] + 1)];
                    const int pos = bs + rk[e];
                    if (be - bs == 1) {
                        k1[pos] = key[e];
                        v1[pos] = val[e];
                        bk[e] = -1;
                    } else {
                        k0[pos] = key[e];
                        rk[e] = pos;
                    }
                }
            }
            __syncthreads();
            UNIT_PH(7);
            // ---- G: rank inside multi-key buckets (equal keys by scatter position)
#pragma unroll
            for (int e = 0; e < EPT; ++e) {
                if (bk[e] >= 0) {
                    const int bs = hist[hidx(bk[e])], be = hist[hidx(bk[e] + 1)];
                    const int32_t kk = key[e];
                    const int pos = rk[e];
                    int rank = 0;
                    for (int q = bs; q < be; ++q) {
                        const int32_t kq = k0[q];
                        rank += (kq < kk) | ((kq == kk) & (q < pos));
                    }
                    k1[bs + rank] = kk;
                    v1[bs + rank] = val[e];
                }
            }
            __syncthreads();
            UNIT_PH(8);
            // ---- H: fp64 segmented reduction over contiguous slices (odd stride: no bank
            //      conflicts); merged entries -> (k0, v0) at their output index, which is also
            //      recorded per head in hist[p] for the row pointers
            const int E2 = ((V + T - 1) / T) | 1;
            const int p0 = min(V, tid * E2), p1 = min(V, p0 + E2);
            int rc = 0;
            if (p0 < p1) {
                int lo = 0, hi = nr;
                while (hi - lo > 1) {
                    const int mid = (lo + hi) >> 1;
                    if (rss[mid] <= p0) lo = mid; else hi = mid;
                }
                rc = lo;
            }
            int nh = 0;
            {
                int r = rc, st = rss[rc], nx = rss[rc + 1];
                for (int p = p0; p < p1; ++p) {
                    while (p >= nx) { ++r; st = nx; nx = rss[r + 1]; }
                    nh += (p == st) || (k1[p] != k1[p - 1]);
                }
            }
            int o = g.excl_sum(nh, sc, &U);
            if (warp_id() == 0 && a.debug != 1) lb_publish(a.status, u, U);
            {
                int r = rc, st = rss[rc], nx = rss[rc + 1];
                for (int p = p0; p < p1; ++p) {
                    while (p >= nx) { ++r; st = nx; nx = rss[r + 1]; }
                    const int32_t kk = k1[p];
                    if (p == st || kk != k1[p - 1]) {
                        double acc = (double)v1[p];
                        for (int q = p + 1; q < nx && k1[q] == kk; ++q) acc += (double)v1[q];
                        k0[o] = kk;
                        v0[o] = (float)acc;
                        hist[p] = o;
                        ++o;
                    }
                }
            }
            __syncthreads();
            if (tid < nr) rout[tid] = rss[tid] < V ? hist[rss[tid]] : U;
            UNIT_PH(9);
        } else {
            // ---- fallback (a bucket of > kBucketMax keys): per-row natural merge sort
            if (tid == 0) atomicAdd(a.n_fallback, 1ull);
#pragma unroll
            for (int e = 0; e < EPT; ++e) {
                const int p = pb + e;
                if (p < n) { k0[p] = key[e]; v0[p] = val[e]; }
            }
            __syncthreads();
            int *bA = hist, *bB = hist + (kUnitCap + 1);
            int o = 0;
            for (int r = 0; r < nr; ++r) {
                const int s = ro[r], L = ro[r + 1] - s, Lv = rv[r];
                if (tid == 0) rout[r] = o;
                if (Lv == 0) continue;
                const int which = natural_merge_sort<NW, 1, kUnitCap>(g, k0 + s, v0 + s, k1 + s, v1 + s, bA, bB, L, sc);
                if (which == 0) {
                    for (int q = tid; q < L; q += T) { k1[s + q] = k0[s + q]; v1[s + q] = v0[s + q]; }
                    __syncthreads();
                }
                // the sorted row is in k1; its merged entries go to k0 at o <= s (dead slots)
                o += segmented_reduce_out<NW, 1>(g, k1 + s, v1 + s, Lv, k0 + o, v0 + o, sc);
                __syncthreads();
            }
            U = o;
            if (warp_id() == 0 && a.debug != 1) lb_publish(a.status, u, U);
        }
        __syncthreads();
        // ---- I: output offset by look-back, row pointers, merged rows
        if (warp_id() == 0) {
            const int64_t P = a.debug == 1 ? S0 : lb_resolve(a.status, u, U);
            if (lane_id() == 0) s_P = P;
        }
        __syncthreads();
        UNIT_PH(10);
        const int64_t P = s_P;
        if (tid < nr) a.crowptr[r0 + tid] = P + rout[tid];
        if (tid == 0 && r1 == a.M) a.crowptr[a.M] = P + U;
        for (int q = tid; q < U; q += T) {
            a.chat_col[P + q] = k0[q];
            a.chat_val[P + q] = v0[q];
        }
        __syncthreads();
        UNIT_PH(11);
    }
    if (prof_on)
        for (int k = 0; k < 16; ++k) atomicAdd(a.prof + k, ph[k]);
}

// Long rows: merged row (side buffer) -> its C position (one CTA per row, 4 loads in flight).
constexpr int kCopyThreads = 256;
__global__ void __launch_bounds__(kCopyThreads) k_copy_long(const int32_t *__restrict__ rows, int64_t nrows,
                                                           const int64_t *__restrict__ crowptr,
                                                           const int64_t *__restrict__ ccount,
                                                           const int64_t *__restrict__ side_off,
                                                           const int32_t *__restrict__ side_col,
                                                           const float *__restrict__ side_val,
                                                           int32_t *__restrict__ out_col, float *__restrict__ out_val) {
    for (int64_t r = blockIdx.x; r < nrows; r += gridDim.x) {
        const int i = rows[r];
        const int64_t P = crowptr[i], U = ccount[i], so = side_off[i];
        for (int64_t q0 = 0; q0 < U; q0 += 4 * kCopyThreads) {
            int32_t c[4];
            float v[4];
#pragma unroll
            for (int j = 0; j < 4; ++j) {
                const int64_t q = q0 + j * kCopyThreads + threadIdx.x;
                if (q < U) { c[j] = __ldcs(side_col + so + q); v[j] = __ldcs(side_val + so + q); }
            }
#pragma unroll
            for (int j = 0; j < 4; ++j) {
                const int64_t q = q0 + j * kCopyThreads + threadIdx.x;
                if (q < U) { out_col[P + q] = c[j]; out_val[P + q] = v[j]; }
            }
        }
    }
}

}  // namespace spg
