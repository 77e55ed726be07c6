// Stage (4): merge of Ĉ into C -- per row, sort by column + segmented reduce.
//
// PAPER.md §IV-D L452-L477 L: "elements with the same indices are merged into unique elements.
// This merging process is highly memory intensive ... B-Limiting ... limiting the number of
// blocks allocated to an SM ... extra shared memory ... applied only to the large rows of ĉ_i*".
// BASELINE.json north_star: "a row-bucketed sort plus segmented reduce into CSR".
//
// Every bin sorts the row's (col, val) pairs by col and reduces equal-col segments in fp64,
// rounding once to fp32; the merged row is written back in place at the head of the row's
// Ĉ bucket and its length to ccount[i].
//
// A row's bucket is a concatenation of runs -- one per stored a_ik, each in B's ascending
// column order -- so the sort is a *natural merge sort*: ascending runs are detected, then
// merged pairwise level by level; each thread produces a contiguous slice of every level's
// output, locating its start by a merge-path binary search.  Rows with R runs need
// ceil(log2 R) levels (C2: 4-10 runs on the rows that hold most products).
//
// Bins (one kernel each): single-run rows are already merged (passthrough); L <= 32 one warp,
// register bitonic network; L <= 256 / L <= 1024 one warp per row, row in the warp's smem
// slice; L <= t_lim (4096) four warps per row; L > t_lim B-Limited (see k_merge_limited).
#pragma once
#include "analysis.cuh"

namespace spg {

constexpr int32_t kKeyPad = 0x7fffffff;
constexpr unsigned kFull = 0xffffffffu;

// ------------------------------------------------------------------------ warp bin ---
__global__ void __launch_bounds__(256) k_merge_warp(const int32_t *__restrict__ rows, int64_t nrows,
                                                    const int64_t *__restrict__ rowoff, int32_t *__restrict__ chat_col,
                                                    float *__restrict__ chat_val, int64_t *__restrict__ ccount,
                                                    const int64_t *__restrict__ crowptr, int32_t *__restrict__ out_col,
                                                    float *__restrict__ out_val) {
    const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    if (gw >= nrows) return;
    const int lane = lane_id();
    const int i = rows[gw];
    const int64_t s = rowoff[i];
    const int L = (int)(rowoff[i + 1] - s);
    int32_t key = lane < L ? chat_col[s + lane] : kKeyPad;
    double v = lane < L ? (double)chat_val[s + lane] : 0.0;
    // bitonic sort of 32 (key, v) pairs, ascending by key
#pragma unroll
    for (int k = 2; k <= 32; k <<= 1) {
#pragma unroll
        for (int j = k >> 1; j > 0; j >>= 1) {
            int32_t pk = __shfl_xor_sync(kFull, key, j);
            double pv = __shfl_xor_sync(kFull, v, j);
            bool up = (lane & k) == 0;
            bool lower = (lane & j) == 0;
            bool take = lower == up ? (pk < key) : (pk > key);
            if (take) { key = pk; v = pv; }
        }
    }
    const int32_t prev = __shfl_up_sync(kFull, key, 1);
    const int32_t next = __shfl_down_sync(kFull, key, 1);
    const bool valid = key != kKeyPad;
    const bool head = lane == 0 || prev != key;
    const unsigned heads = __ballot_sync(kFull, head);
    const int seg_start = 31 - __clz(heads & (lanemask_lt() | (1u << lane)));
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
        double o = __shfl_up_sync(kFull, v, d);
        if (lane - d >= seg_start) v += o;
    }
    const bool tail = valid && (lane == 31 || next != key);
    const unsigned tails = __ballot_sync(kFull, tail);
    if (tail) {
        const int pos = __popc(tails & lanemask_lt());
        if (out_col) {
            const int64_t o = crowptr[i];
            out_col[o + pos] = key;
            out_val[o + pos] = (float)v;
        } else {
            chat_col[s + pos] = key;
            chat_val[s + pos] = (float)v;
        }
    }
    if (lane == 0 && !out_col) ccount[i] = __popc(tails);
}


// ------------------------------------------------------------------ thread groups ---
// A group of NW warps works on one row; GROUPS groups share a CTA.  Groups synchronise with
// __syncwarp (NW = 1), __syncthreads (one group per CTA) or a named barrier (bar.sync id, n).
template <int NW, int GROUPS>
struct Group {
    static constexpr int T = NW * 32;
    int gid, gtid;
    __device__ __forceinline__ Group() : gid(threadIdx.x / T), gtid(threadIdx.x % T) {}
    __device__ __forceinline__ void sync() const {
        if constexpr (NW == 1) __syncwarp();
        else if constexpr (GROUPS == 1) __syncthreads();
        else asm volatile("bar.sync %0, %1;" ::"r"(1 + gid), "r"(T) : "memory");
    }
    // exclusive prefix sum over the group; `sc` = NW + 1 ints private to the group
    __device__ __forceinline__ int excl_sum(int v, int *sc, int *total) const {
        const int inc = warp_incl_sum(v);
        if constexpr (NW == 1) {
            *total = __shfl_sync(kFull, inc, 31);
            return inc - v;
        } else {
            const int w = gtid >> 5;
            if (lane_id() == 31) sc[w] = inc;
            sync();
            if (gtid == 0) {
                int run = 0;
                for (int q = 0; q < NW; ++q) { const int t = sc[q]; sc[q] = run; run += t; }
                sc[NW] = run;
            }
            sync();
            const int r = sc[w] + inc - v;
            *total = sc[NW];
            sync();
            return r;
        }
    }
    __device__ __forceinline__ int reduce_min(int v, int *sc) const {
        v = warp_min(v);
        if constexpr (NW == 1) return v;
        else {
            if (lane_id() == 0) sc[gtid >> 5] = v;
            sync();
            int r = sc[0];
            for (int q = 1; q < NW; ++q) r = min(r, sc[q]);
            sync();
            return r;
        }
    }
    // excl_sum with a single barrier: every thread combines the warp totals itself.  The caller
    // guarantees a group barrier between these reads of sc[0, NW) and the next write to them.
    __device__ __forceinline__ int excl_sum1(int v, int *sc, int *total) const {
        const int inc = warp_incl_sum(v);
        if constexpr (NW == 1) {
            *total = __shfl_sync(kFull, inc, 31);
            return inc - v;
        } else {
            const int w = gtid >> 5;
            if (lane_id() == 31) sc[w] = inc;
            sync();
            int before = 0, tot = 0;
            if constexpr (NW <= 8) {
#pragma unroll
                for (int q = 0; q < NW; ++q) {
                    const int t = sc[q];
                    before += q < w ? t : 0;
                    tot += t;
                }
            } else {
                const int t = lane_id() < NW ? sc[lane_id()] : 0;
                const int ci = warp_incl_sum(t);
                before = __shfl_sync(kFull, ci - t, w);
                tot = __shfl_sync(kFull, ci, NW - 1);
            }
            *total = tot;
            return before + inc - v;
        }
    }
    // min and max in one shared-memory round; `sc` needs 2 * NW + 1 ints
    __device__ __forceinline__ void reduce_minmax(int &mn, int &mx, int *sc) const {
        mn = warp_min(mn);
        mx = warp_max(mx);
        if constexpr (NW > 1) {
            if (lane_id() == 0) { sc[gtid >> 5] = mn; sc[NW + 1 + (gtid >> 5)] = mx; }
            sync();
            int a = sc[0], b = sc[NW + 1];
            for (int q = 1; q < NW; ++q) { a = min(a, sc[q]); b = max(b, sc[NW + 1 + q]); }
            sync();
            mn = a;
            mx = b;
        }
    }
    __device__ __forceinline__ int reduce_max(int v, int *sc) const {
        v = warp_max(v);
        if constexpr (NW == 1) return v;
        else {
            if (lane_id() == 0) sc[gtid >> 5] = v;
            sync();
            int r = sc[0];
            for (int q = 1; q < NW; ++q) r = max(r, sc[q]);
            sync();
            return r;
        }
    }
};

__device__ __forceinline__ void cp_async4(void *smem_dst, const void *gmem_src) {
    const unsigned d = (unsigned)__cvta_generic_to_shared(smem_dst);
    asm volatile("cp.async.ca.shared.global [%0], [%1], 4;" ::"r"(d), "l"(gmem_src) : "memory");
}
__device__ __forceinline__ void cp_async_wait_all() { asm volatile("cp.async.wait_all;" ::: "memory"); }

// Smem footprint of a sorter with capacity CAP: keys/vals double-buffered + run bounds.
template <int CAP>
struct SortSmem {
    static constexpr int kBoundsA = CAP + 1, kBoundsB = CAP / 2 + 2;
    static constexpr int kBytes = CAP * 16 + (kBoundsA + kBoundsB) * 4;
};

// Natural merge sort of k[0..L) (with v) held in smem by group g.  Returns 0 if the sorted
// data ends in (k0, v0), 1 if in (k1, v1).
template <int NW, int GROUPS, int CAP>
__device__ __forceinline__ int natural_merge_sort(const Group<NW, GROUPS> &g, int32_t *k0, float *v0, int32_t *k1,
                                                  float *v1, int *bA, int *bB, int L, int *sc) {
    constexpr int T = NW * 32;
    const int E = ((L + T - 1) / T) | 1;
    const int p0 = min(L, g.gtid * E), p1 = min(L, p0 + E);
    // run heads: p == 0 or k[p] <= k[p-1]
    int nh = 0;
    for (int p = p0; p < p1; ++p) nh += (p == 0 || k0[p] <= k0[p - 1]);
    int R;
    int pos = g.excl_sum(nh, sc, &R);
    for (int p = p0; p < p1; ++p)
        if (p == 0 || k0[p] <= k0[p - 1]) bA[pos++] = p;
    if (g.gtid == 0) bA[R] = L;
    g.sync();
    int32_t *ks = k0, *kd = k1;
    float *vs = v0, *vd = v1;
    int *bs = bA, *bd = bB;
    int which = 0;
    while (R > 1) {
        const int pairs = (R + 1) >> 1;
        if (p0 < p1) {
            int lo = 0, hi = pairs;          // pair q: last q with bs[2q] <= p0
            while (hi - lo > 1) {
                const int mid = (lo + hi) >> 1;
                if (bs[2 * mid] <= p0) lo = mid; else hi = mid;
            }
            int q = lo;
            int o = p0;
            while (o < p1) {
                const int a0 = bs[2 * q];
                const int a1 = bs[min(2 * q + 1, R)];
                const int b1 = bs[min(2 * q + 2, R)];
                const int na = a1 - a0, nb = b1 - a1;
                const int d = o - a0;
                int ilo = max(0, d - nb), ihi = min(d, na);
                while (ilo < ihi) {           // merge path: first i with A[i] > B[d-i-1]
                    const int mi = (ilo + ihi) >> 1;
                    if (ks[a0 + mi] <= ks[a1 + d - mi - 1]) ilo = mi + 1; else ihi = mi;
                }
                int ia = ilo, jb = d - ilo;
                int32_t ka = ia < na ? ks[a0 + ia] : kKeyPad;
                float va = ia < na ? vs[a0 + ia] : 0.f;
                int32_t kb = jb < nb ? ks[a1 + jb] : kKeyPad;
                float vb = jb < nb ? vs[a1 + jb] : 0.f;
                const int oend = min(p1, b1);
                for (; o < oend; ++o) {
                    const bool tA = jb >= nb || (ia < na && ka <= kb);
                    kd[o] = tA ? ka : kb;
                    vd[o] = tA ? va : vb;
                    ia += tA;
                    jb += !tA;
                    const bool ok = tA ? ia < na : jb < nb;
                    const int idx = tA ? a0 + ia : a1 + jb;
                    const int32_t nk = ok ? ks[idx] : kKeyPad;
                    const float nv = ok ? vs[idx] : 0.f;
                    if (tA) { ka = nk; va = nv; } else { kb = nk; vb = nv; }
                }
                ++q;
            }
        }
        g.sync();
        for (int q = g.gtid; q <= pairs; q += T) bd[q] = q < pairs ? bs[2 * q] : L;
        g.sync();
        { int32_t *t = ks; ks = kd; kd = t; }
        { float *t = vs; vs = vd; vd = t; }
        { int *t = bs; bs = bd; bd = t; }
        which ^= 1;
        R = pairs;
    }
    return which;
}

// Segmented reduce of a sorted row in smem; writes the merged row to out_col/out_val[0..U)
// and returns U.  Each thread owns a contiguous slice; a segment is summed in fp64 by the
// thread owning its head.
template <int NW, int GROUPS>
__device__ __forceinline__ int segmented_reduce_out(const Group<NW, GROUPS> &g, const int32_t *k, const float *v,
                                                    int L, int32_t *__restrict__ out_col, float *__restrict__ out_val,
                                                    int *sc) {
    constexpr int T = NW * 32;
    const int E = ((L + T - 1) / T) | 1;
    const int p0 = min(L, g.gtid * E), p1 = min(L, p0 + E);
    int nh = 0;
    for (int p = p0; p < p1; ++p) nh += (p == 0 || k[p] != k[p - 1]);
    int total;
    int pos = g.excl_sum(nh, sc, &total);
    for (int p = p0; p < p1; ++p) {
        if (p == 0 || k[p] != k[p - 1]) {
            const int32_t key = k[p];
            double acc = (double)v[p];
            for (int q = p + 1; q < L && k[q] == key; ++q) acc += (double)v[q];
            out_col[pos] = key;
            out_val[pos] = (float)acc;
            ++pos;
        }
    }
    return total;
}

// ------------------------------------------------------------- bucket sort + reduce ---
// MSD counting sort of one row by a group of T threads, then fp64 segmented reduction:
//   1. each thread loads EPT elements (striped) into registers; min/max of the columns;
//   2. nb = 2^ceil(log2 L) buckets over the column span, bucket = (col - min) >> sh;
//      histogram with shared-memory integer atomics, exclusive scan (each thread owns a
//      contiguous range of buckets);
//   3. scatter by atomic rank into dk/dv; every bucket now holds the keys of a 2^sh-wide
//      column range (on average < 2 elements), finished by an insertion sort;
//   4. each thread walks its buckets in order and reduces equal columns in fp64, compacting
//      in place inside its own bucket range; warps then copy their contiguous output slice
//      to global memory with coalesced stores.
// Equal columns always share a bucket, so no segment crosses a thread's range.  A bucket with
// more than kBucketMax entries (many distinct columns packed into a narrow range) makes the
// function return -1 before anything is written; the caller falls back to the natural merge sort.
#ifndef SPG_BUCKET_MAX
#define SPG_BUCKET_MAX 127   // (<= 127: the sort code keeps 7 bits of atomic rank; 64: C3 +5.4 ms)
#endif
constexpr int kBucketMax = SPG_BUCKET_MAX;
static_assert(kBucketMax <= 127, "sort codes hold 7 bits of in-bucket rank");
#ifndef SPG_BIN_THREADS_SM
#define SPG_BIN_THREADS_SM 1024   // k_merge_bucket: 64 registers, no spills (1280: C5 +0.5 ms)
#endif
#ifndef SPG_LIM_LS
#define SPG_LIM_LS 0   // (A/B build knob: 1 = twice the buckets in the B-Limited sorts, capped at 16384)
#endif
#ifndef SPG_LIM_GPIPE
#define SPG_LIM_GPIPE 0   // (A/B build knob: software-pipelined B-Limited group sorts)
#endif
#ifndef SPG_SCATTER_BALLOT
#define SPG_SCATTER_BALLOT 0   // (A/B build knob: coarse scatter by per-group ballots when a warp spans < 4 groups)
#endif
#ifndef SPG_LIM_T78
#define SPG_LIM_T78 1   // coarse groups up to 7/8 of the sorter when every bin is small (C5 limited 63.6 -> 62.6 ms)
#endif
#ifndef SPG_LIM_UNR2
#define SPG_LIM_UNR2 false   // B-Limited groups: one code per ranking step (two: C5 limited merge 63.6 -> 67.5 ms)
#endif
#ifndef SPG_BIN_UNR2
#define SPG_BIN_UNR2 false   // regular bins: one code per ranking step (two: C2 merge 4.68 -> 5.62 ms)
#endif

__device__ __forceinline__ int nextpow2_log(int x) { return x <= 1 ? 0 : 32 - __clz(x - 1); }

// histogram slot of bucket b: one pad word per 32 buckets, so threads walking contiguous bucket
// ranges (stride = buckets per thread) hit distinct banks
#ifndef SPG_HPAD
#define SPG_HPAD 1   // (A/B build knob: 0 = no pad word)
#endif
__host__ __device__ __forceinline__ constexpr int hidx(int b) { return SPG_HPAD ? b + (b >> 5) : b; }

// striped load of a row into registers (slot gtid + e*T); sentinel (padding) entries stay kKeyPad
template <int NW, int GROUPS, int EPT>
__device__ __forceinline__ void bsr_load(const Group<NW, GROUPS> &g, const int32_t *sk, const float *sv, int L,
                                         int32_t (&key)[EPT], float (&val)[EPT]) {
    constexpr int T = NW * 32;
#pragma unroll
    for (int e = 0; e < EPT; ++e) {
        const int p = g.gtid + e * T;
        key[e] = p < L ? sk[p] : kKeyPad;
        val[e] = p < L ? sv[p] : 0.f;
    }
}

template <int NW, int GROUPS, int EPT, int LS = 0, bool UNR2 = false, int PRECLEAR = 0>
__device__ __forceinline__ int bucket_sort_reduce_regs(const Group<NW, GROUPS> &g, int32_t (&key)[EPT],
                                                       float (&val)[EPT], int L, int32_t *dk, float *dv, int32_t *dk2,
                                                       float *dv2, int *hist, int32_t *out_col, float *out_val,
                                                       int *sc, int32_t pmn = 1, int32_t pmx = 0);


// LS: buckets = 2^LS x (slots rounded up to a power of two); more buckets, fewer shared ones.
// UNR2: in-bucket ranking two keys per step (the B-Limited groups' wider buckets: C3 -5 %; the
// regular bins' mostly 2-key buckets are faster without)
template <int NW, int GROUPS, int EPT, int LS = 0, bool UNR2 = false>
__device__ __forceinline__ int bucket_sort_reduce(const Group<NW, GROUPS> &g, const int32_t *sk, const float *sv,
                                                  int L, int32_t *dk, float *dv, int32_t *dk2, float *dv2,
                                                  int *hist, int32_t *out_col, float *out_val, int *sc,
                                                  int32_t pmn = 1, int32_t pmx = 0) {
    int32_t key[EPT];
    float val[EPT];
    bsr_load<NW, GROUPS, EPT>(g, sk, sv, L, key, val);
    return bucket_sort_reduce_regs<NW, GROUPS, EPT, LS, UNR2>(g, key, val, L, dk, dv, dk2, dv2, hist, out_col, out_val,
                                                              sc, pmn, pmx);
}

// the row already in registers (bsr_load; software-pipelined callers load the next row early)
template <int NW, int GROUPS, int EPT, int LS, bool UNR2, int PRECLEAR>
__device__ __forceinline__ int bucket_sort_reduce_regs(const Group<NW, GROUPS> &g, int32_t (&key)[EPT],
                                                       float (&val)[EPT], int L, int32_t *dk, float *dv, int32_t *dk2,
                                                       float *dv2, int *hist, int32_t *out_col, float *out_val,
                                                       int *sc, int32_t pmn, int32_t pmx) {
    constexpr int T = NW * 32;
    int32_t mn = pmn, mx = pmx;
    if (pmn > pmx) {   // no exact column range from the plan (rowmn / rowmx): reduce it here
        mn = kKeyPad;
        mx = 0;
#pragma unroll
        for (int e = 0; e < EPT; ++e)
            if (key[e] != kKeyPad) { mn = min(mn, key[e]); mx = max(mx, key[e]); }
        g.reduce_minmax(mn, mx, sc);
    }
    const uint32_t span = (uint32_t)(mx - mn);
    // (>= 64 buckets: sh <= 25, so a key's in-bucket bits and its 7-bit atomic rank fit 32 bits)
    const int lognb = LS > 0 ? min(14, max(6, nextpow2_log(L) + LS)) : max(6, nextpow2_log(L));   // (LS: <= 16384 buckets)
    const int nb = 1 << lognb;
    const int bits = span ? 32 - __clz(span) : 0;
    const int sh = max(0, bits - lognb);
    const uint32_t lowmask = (1u << sh) - 1u;
    // PRECLEAR > 0: the caller zeroed hist[0, PRECLEAR] (and the previous row cleared it after its
    // ranking), so the row starts with its atomics -- one barrier less per row
    if constexpr (PRECLEAR == 0) {
        for (int b = g.gtid; b <= hidx(nb); b += T) hist[b] = 0;
        g.sync();
    }
    // one shared atomic per element (spread-address ATOMS cost ~2 cycles per lane): its return
    // value is the element's rank inside its bucket, reused by the scatter below
    int rk[EPT];
#pragma unroll
    for (int e = 0; e < EPT; ++e)
        rk[e] = key[e] != kKeyPad ? atomicAdd(&hist[hidx((key[e] - mn) >> sh)], 1) : 0;
    g.sync();
    const int bpt = (nb + T - 1) / T;
    const int b0 = min(nb, g.gtid * bpt), b1 = min(nb, b0 + bpt);
    int cnt = 0, mxc = 0;
    for (int b = b0; b < b1; ++b) {
        const int c = hist[hidx(b)];
        cnt += c;
        mxc = max(mxc, c);
    }
    // (an over-full bucket adds 2^16 to the total: the overflow test rides on the scan.  A row holds
    // at most 9216 < 2^16 slots and a group at most 1024 threads, so the flagged total stays below
    // 2^26 + 2^16 and cannot wrap, and any flag lifts it above every real count)
    static_assert(NW * 32 <= 1024, "overflow flag sized for <= 1024 threads");
    int tot;
    int ex = g.excl_sum(cnt + (mxc > kBucketMax ? (1 << 16) : 0), sc, &tot);
    if (tot >= (1 << 16)) {
        if constexpr (PRECLEAR > 0) {   // (the cnt reads above are behind the scan's barriers)
            for (int b = g.gtid; b <= PRECLEAR; b += T) hist[b] = 0;
            g.sync();
        }
        return -1;
    }
    for (int b = b0; b < b1; ++b) {
        const int c = hist[hidx(b)];
        hist[hidx(b)] = ex;
        ex += c;
    }
    if (g.gtid == 0) hist[hidx(nb)] = tot;
    g.sync();
    // 1. scatter: bucket start + atomic rank (unordered inside a bucket).  What is scattered is the
    //    element's in-bucket sort code c = (key's low sh bits) << 7 | atomic rank: the keys of one
    //    bucket share their high bits, so c orders them by key, ties by scatter order, and is unique
    //    (ranks < 2^7: buckets above kBucketMax took the fallback)
    int pos[EPT];
    uint32_t *dc = reinterpret_cast<uint32_t *>(dk);
#pragma unroll
    for (int e = 0; e < EPT; ++e) {
        pos[e] = -1;
        if (key[e] != kKeyPad) {
            pos[e] = hist[hidx((key[e] - mn) >> sh)] + rk[e];
            dc[pos[e]] = ((((uint32_t)(key[e] - mn)) & lowmask) << 7) | (uint32_t)rk[e];
        }
    }
    g.sync();
    // 2. bucket b = [hist[b], hist[b+1]).  Every element counts the codes of its bucket below its own
    //    (one load and one compare per key) and moves to its sorted slot.
#pragma unroll
    for (int e = 0; e < EPT; ++e) {
        if (pos[e] >= 0) {
            const int b = (key[e] - mn) >> sh;
            const int bs = hist[hidx(b)], be = hist[hidx(b + 1)];
            const uint32_t ce = ((((uint32_t)(key[e] - mn)) & lowmask) << 7) | (uint32_t)rk[e];
            int rank = 0;
            if (be - bs > 1) {   // (a bucket of one key is already in place)
                int q = bs;
                if constexpr (UNR2)
                    for (; q + 1 < be; q += 2) rank += (dc[q] < ce) + (dc[q + 1] < ce);
                for (; q < be; ++q) rank += dc[q] < ce;
            }
            dk2[bs + rank] = key[e];
            dv2[bs + rank] = val[e];
        }
    }
    g.sync();
    if constexpr (PRECLEAR > 0)   // hist's last reads (the ranking) are done: clear it for the next row
        for (int b = g.gtid; b <= PRECLEAR; b += T) hist[b] = 0;
    // 3. segmented reduction over contiguous slices (fp64), compacted into (dk, dv)
    L = tot;   // valid (non-sentinel) entries
    const int E = ((L + T - 1) / T) | 1;     // odd stride between thread slices: no bank conflicts
    const int p0 = min(L, g.gtid * E), p1 = min(L, p0 + E);
    const int32_t before = p0 > 0 && p0 < L ? dk2[p0 - 1] : -1;   // (-1 is no column)
    int nh = 0;
    {
        int32_t prevk = before;
        for (int p = p0; p < p1; ++p) {
            const int32_t k = dk2[p];
            nh += k != prevk;
            prevk = k;
        }
    }
    int U;
    int o = g.excl_sum1(nh, sc, &U);
    {   // a segment continuing from the previous slice is summed by that slice's thread
        int32_t prevk = before, cur = -1;
        double acc = 0.0;
        for (int p = p0; p < p1; ++p) {
            const int32_t k = dk2[p];
            const float v = dv2[p];
            if (k != prevk) {
                if (cur != -1) { dk[o] = cur; dv[o] = (float)acc; ++o; }
                cur = k;
                acc = (double)v;
            } else if (cur != -1) {
                acc += (double)v;
            }
            prevk = k;
        }
        if (cur != -1) {
            for (int q = p1; q < L && dk2[q] == cur; ++q) acc += (double)dv2[q];
            dk[o] = cur;
            dv[o] = (float)acc;
        }
    }
    g.sync();
    // 4. coalesced copy of the merged row
    for (int q = g.gtid; q < U; q += T) {
        out_col[q] = dk[q];
        out_val[q] = dv[q];
    }
    return U;
}

constexpr int ceil_pow2(int x) { return x <= 1 ? 1 : 2 * ceil_pow2((x + 1) / 2); }

template <int NW, int EPT, int LS = 0>
struct BucketSmem {
    static constexpr int kCap = NW * 32 * EPT;
    static constexpr int kNb = ceil_pow2(kCap) << LS;
    static constexpr int kBytes = kCap * 16 + (hidx(kNb) + 4) * 4;
};

// Rows of one bin: bucket sort per row; rows whose buckets overflow go to a fallback list.
template <int NW, int GROUPS, int EPT, int LS = 0>
__global__ void __launch_bounds__(NW * 32 * GROUPS, SPG_BIN_THREADS_SM / (NW * 32 * GROUPS)) k_merge_bucket(const int32_t *__restrict__ rows, int64_t nrows,
                                                                  const int64_t *__restrict__ rowoff,
                                                                  int32_t *__restrict__ chat_col,
                                                                  float *__restrict__ chat_val,
                                                                  int64_t *__restrict__ ccount,
                                                                  int32_t *__restrict__ fb_rows,
                                                                  unsigned *__restrict__ fb_count, int64_t cap_skip,
                                                                  const int64_t *__restrict__ crowptr,
                                                                  int32_t *__restrict__ out_col,
                                                                  float *__restrict__ out_val,
                                                                  const int32_t *__restrict__ rowmn,
                                                                  const int32_t *__restrict__ rowmx) {
    using S = BucketSmem<NW, EPT, LS>;
    extern __shared__ __align__(16) unsigned char smem_raw[];
    __shared__ int sc_all[GROUPS][2 * NW + 2];
    const Group<NW, GROUPS> g;
    unsigned char *slice = smem_raw + (size_t)g.gid * S::kBytes;
    int32_t *dk = (int32_t *)slice;
    float *dv = (float *)(slice + S::kCap * 4);
    int32_t *dk2 = (int32_t *)(slice + S::kCap * 8);
    float *dv2 = (float *)(slice + S::kCap * 12);
    int *hist = (int *)(slice + S::kCap * 16);
    for (int64_t r = (int64_t)blockIdx.x * GROUPS + g.gid; r < nrows; r += (int64_t)gridDim.x * GROUPS) {
        const int i = rows[r];
        const int64_t s = rowoff[i];
        const int L = (int)(rowoff[i + 1] - s);
        if (L > S::kCap) continue;          // (limited list) rows above this kernel's capacity
        const int64_t o = out_col ? crowptr[i] : s;
        const int U = bucket_sort_reduce<NW, GROUPS, EPT, LS, SPG_BIN_UNR2>(g, chat_col + s, chat_val + s, L, dk, dv, dk2, dv2, hist,
                                                          (out_col ? out_col : chat_col) + o,
                                                          (out_col ? out_val : chat_val) + o, sc_all[g.gid],
                                                          rowmn ? rowmn[i] : 1, rowmn ? rowmx[i] : 0);
        if (g.gtid == 0) {
            if (U >= 0) ccount[i] = U;
            else if (fb_rows) fb_rows[atomicAdd(fb_count, 1u)] = i;
            else ccount[i] = -1;   // limited list: k_merge_limited takes the row (merge-path fallback)
        }
        // (no barrier: the next row first writes hist, whose last reads -- the ranking -- and
        // those of sc are behind the reduction phase's barriers; dk / dv, read by the copy-out,
        // are next written after two more barriers)
    }
    (void)cap_skip;
}

// Software-pipelined variant (in place): per row r of the bin the group holds row r's slots in
// registers, loads row r + S (S = groups in the grid) while sorting row r, and row r + 2S's
// (offset, length, id) from the bin's meta table -- one independent load -- so neither the
// row data nor its offsets are a dependent memory round trip on the sort's critical path.
struct RowMeta {
    int64_t s;    // first slot of the row's Ĉ bucket
    int32_t L;    // padded length
    int32_t i;    // row id
    int32_t Lv;   // products (valid slots)
    int32_t pad;
};

__global__ void k_row_meta(const int32_t *__restrict__ order, int64_t n, const int64_t *__restrict__ rowoff,
                           const int64_t *__restrict__ rowwork, const int32_t *__restrict__ rowmn,
                           const int32_t *__restrict__ rowmx, RowMeta *__restrict__ meta,
                           int2 *__restrict__ rng) {
    for (int64_t q = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; q < n; q += (int64_t)gridDim.x * blockDim.x) {
        const int i = order[q];
        const int64_t s = rowoff[i];
        meta[q] = RowMeta{s, (int32_t)(rowoff[i + 1] - s), i, (int32_t)rowwork[i], 0};
        // exact column range of the row (mn > mx: unknown), apart from the meta table: loaded
        // per row at the top of the pipelined loop instead of held three rows ahead in registers
        if (rng) rng[q] = rowmn ? make_int2(rowmn[i], rowmx[i]) : make_int2(1, 0);
    }
}

template <int NW, int GROUPS, int EPT, int LS = 0>
__global__ void __launch_bounds__(NW * 32 * GROUPS, 1024 / (NW * 32 * GROUPS)) k_merge_bucket_pipe(
    const RowMeta *__restrict__ meta, int64_t nrows, int32_t *__restrict__ chat_col, float *__restrict__ chat_val,
    int64_t *__restrict__ ccount, int32_t *__restrict__ fb_rows, unsigned *__restrict__ fb_count,
    const int2 *__restrict__ rng) {
    using S = BucketSmem<NW, EPT, LS>;
    extern __shared__ __align__(16) unsigned char smem_raw[];
    __shared__ int sc_all[GROUPS][2 * NW + 2];
    const Group<NW, GROUPS> g;
    unsigned char *slice = smem_raw + (size_t)g.gid * S::kBytes;
    int32_t *dk = (int32_t *)slice;
    float *dv = (float *)(slice + S::kCap * 4);
    int32_t *dk2 = (int32_t *)(slice + S::kCap * 8);
    float *dv2 = (float *)(slice + S::kCap * 12);
    int *hist = (int *)(slice + S::kCap * 16);
    const int64_t stride = (int64_t)gridDim.x * GROUPS;
    int64_t r = (int64_t)blockIdx.x * GROUPS + g.gid;
    const RowMeta none{0, 0, -1, 0, 0};
    RowMeta m0 = r < nrows ? meta[r] : none;
    RowMeta m1 = r + stride < nrows ? meta[r + stride] : none;
    int32_t key[EPT];
    float val[EPT];
    bsr_load<NW, GROUPS, EPT>(g, chat_col + m0.s, chat_val + m0.s, m0.L <= S::kCap ? m0.L : 0, key, val);
    // PRECLEAR: hist starts zeroed, every row leaves it zeroed
    for (int b = g.gtid; b <= hidx(S::kNb); b += NW * 32) hist[b] = 0;
    g.sync();
    while (r < nrows) {
        const int2 rg = rng ? rng[r] : make_int2(1, 0);
        int32_t kn[EPT];
        float vn[EPT];
        bsr_load<NW, GROUPS, EPT>(g, chat_col + m1.s, chat_val + m1.s, m1.L <= S::kCap ? m1.L : 0, kn, vn);
        const RowMeta m2 = r + 2 * stride < nrows ? meta[r + 2 * stride] : none;
        if (m0.L <= S::kCap) {
            const int U = bucket_sort_reduce_regs<NW, GROUPS, EPT, LS, SPG_BIN_UNR2, hidx(S::kNb)>(
                g, key, val, m0.L, dk, dv, dk2, dv2, hist, chat_col + m0.s, chat_val + m0.s, sc_all[g.gid], rg.x, rg.y);
            if (g.gtid == 0) {
                if (U >= 0) ccount[m0.i] = U;
                else if (fb_rows) fb_rows[atomicAdd(fb_count, 1u)] = m0.i;
                else ccount[m0.i] = -1;   // limited list: k_merge_limited takes the row
            }
        }
        // (no barrier needed between rows, see k_merge_bucket)
#pragma unroll
        for (int e = 0; e < EPT; ++e) { key[e] = kn[e]; val[e] = vn[e]; }
        m0 = m1;
        m1 = m2;
        r += stride;
    }
}


// -------------------------------------------- warp merge-path natural merge sort (WMP) ---
// No shared-memory atomics (see k_count_rows).  A row's bucket is a concatenation of runs (one
// per stored a_ik, ascending, sentinel-padded to 8 slots), so it is sorted by merging them.
// A group of NW warps (T = 32*NW threads) per row:
//   1. 16-byte vector loads; (col, val) packed into one u64 (col in the high word) in smem;
//      runs start at vector boundaries where the column descends (or the previous run ended
//      in sentinels), found per vector and compacted in order (ballot / group scan);
//   2. levels of pairwise merges, ping-ponging between two smem buffers: thread t produces the
//      t-th slice of each level's output, locating its start in the pair by a merge-path search
//      and merging with a branch-free loop (one predicated LDS per output; keys compared as
//      32-bit integers, ties taken from the left run);
//   3. reduction: each warp walks its share of the sorted products 32 at a time (shares start
//      at segment heads): heads by neighbour compare, fp64 sums of duplicates, ballot-compacted
//      output, straight to the output (NW = 1) or staged per warp in smem and copied out at the
//      warp's scanned offset (NW > 1); output = C at crowptr[i] or in place in Ĉ.
__device__ __forceinline__ uint64_t pack_kv(int32_t k, float v) {
    return ((uint64_t)(uint32_t)k << 32) | (uint64_t)__float_as_uint(v);
}
__device__ __forceinline__ int32_t kv_key(uint64_t x) { return (int32_t)(x >> 32); }
__device__ __forceinline__ float kv_val(uint64_t x) { return __uint_as_float((uint32_t)x); }
constexpr uint64_t kKvMax = 0x7fffffffffffffffull;   // key INT32_MAX: after every product

template <int CAP>
struct WmpSmem {
    static constexpr int kRuns = CAP / 4 + 2;
    static constexpr int kBytes = CAP * 16 + 2 * kRuns * 4;
};


// Software-pipelined warp merge-path bin (rows of <= 256 slots, one warp per row, in place):
// a warp holds the next row's slots (2 vectors per lane) in registers and the row after that's
// (offset, length, id) from the meta table while it merges the current row -- C4's 2M rows of
// 8 runs x 8 were one dependent memory round trip chain per row.
template <int GROUPS>
__global__ void __launch_bounds__(32 * GROUPS) k_merge_wmp_pipe(const RowMeta *__restrict__ meta, int64_t nrows,
                                                                int32_t *__restrict__ chat_col,
                                                                float *__restrict__ chat_val,
                                                                int64_t *__restrict__ ccount) {
    constexpr int CAP = 256;
    using S = WmpSmem<CAP>;
    extern __shared__ __align__(16) unsigned char smem_raw[];
    const int gid = threadIdx.x >> 5, lane = lane_id();
    unsigned char *slice = smem_raw + (size_t)gid * S::kBytes;
    uint64_t *bufA = (uint64_t *)slice;
    uint64_t *bufB = bufA + CAP;
    int *runsA = (int *)(bufB + CAP);
    int *runsB = runsA + S::kRuns;
    const unsigned lt = lanemask_lt();
    const int64_t stride = (int64_t)gridDim.x * GROUPS;
    int64_t r = (int64_t)blockIdx.x * GROUPS + gid;
    const RowMeta none{0, 0, -1, 0, 0};
    RowMeta m0 = r < nrows ? meta[r] : none;
    RowMeta m1 = r + stride < nrows ? meta[r + stride] : none;
    auto load = [&](const RowMeta &m, int4 (&c)[2], float4 (&f)[2]) {
        const int nv = m.L >> 2;
#pragma unroll
        for (int u = 0; u < 2; ++u) {
            const int v = 32 * u + lane;
            c[u] = make_int4(kKeyPad, kKeyPad, kKeyPad, kKeyPad);
            f[u] = make_float4(0.f, 0.f, 0.f, 0.f);
            if (v < nv) {
                c[u] = __ldcs(reinterpret_cast<const int4 *>(chat_col + m.s) + v);
                f[u] = __ldcs(reinterpret_cast<const float4 *>(chat_val + m.s) + v);
            }
        }
    };
    int4 c[2];
    float4 f[2];
    load(m0, c, f);
    while (r < nrows) {
        int4 cn[2];
        float4 fn[2];
        load(m1, cn, fn);
        const RowMeta m2 = r + 2 * stride < nrows ? meta[r + 2 * stride] : none;
        const int Lp = m0.L, Lv = m0.Lv, nv = Lp >> 2;
        // 1. pack + run starts (a run starts where a vector's first key is below the previous key)
        int R = 0;
        {
            int32_t carry = kKeyPad;
#pragma unroll
            for (int u = 0; u < 2; ++u) {
                const int v = 32 * u + lane;
                int32_t prev = __shfl_up_sync(kFull, c[u].w, 1);
                if (lane == 0) prev = carry;
                carry = __shfl_sync(kFull, c[u].w, 31);
                const bool start = v < nv && (v == 0 || c[u].x < prev);
                const unsigned m = __ballot_sync(kFull, start);
                if (start) runsA[R + __popc(m & lt)] = 4 * v;
                R += __popc(m);
                if (v < nv) {
                    ulonglong2 *d = reinterpret_cast<ulonglong2 *>(bufA + 4 * v);
                    d[0] = make_ulonglong2(pack_kv(c[u].x, f[u].x), pack_kv(c[u].y, f[u].y));
                    d[1] = make_ulonglong2(pack_kv(c[u].z, f[u].z), pack_kv(c[u].w, f[u].w));
                }
            }
            if (lane == 0) runsA[R] = Lp;
            __syncwarp();
        }
        // 2. merge levels (merge path per lane over E consecutive outputs)
        uint64_t *src = bufA, *dst = bufB;
        int *rs = runsA, *rd = runsB;
        const int E = (Lp + 31) / 32;
        while (R > 1) {
            const int npairs = (R + 1) >> 1;
            int o = min(Lp, lane * E);
            const int oend = min(Lp, o + E);
            if (o < oend) {
                int lo = 0, hi = npairs;
                while (hi - lo > 1) {
                    const int mid = (lo + hi) >> 1;
                    if (rs[2 * mid] <= o) lo = mid; else hi = mid;
                }
                int q = lo;
                while (o < oend) {
                    const int a0 = rs[2 * q], a1 = rs[min(2 * q + 1, R)], b1 = rs[min(2 * q + 2, R)];
                    const int d = o - a0;
                    int ilo = max(0, d - (b1 - a1)), ihi = min(d, a1 - a0);
                    while (ilo < ihi) {
                        const int mi = (ilo + ihi) >> 1;
                        if (kv_key(src[a0 + mi]) <= kv_key(src[a1 + d - mi - 1])) ilo = mi + 1; else ihi = mi;
                    }
                    int ia = a0 + ilo, jb = a1 + d - ilo;
                    uint64_t xa = ia < a1 ? src[ia] : kKvMax;
                    uint64_t xb = jb < b1 ? src[jb] : kKvMax;
                    const int pend = min(oend, b1);
                    for (; o < pend; ++o) {
                        const bool tA = kv_key(xa) <= kv_key(xb);
                        dst[o] = tA ? xa : xb;
                        const int nxt = tA ? ia + 1 : jb + 1;
                        const uint64_t y = nxt < (tA ? a1 : b1) ? src[nxt] : kKvMax;
                        ia = tA ? nxt : ia;
                        jb = tA ? jb : nxt;
                        xa = tA ? y : xa;
                        xb = tA ? xb : y;
                    }
                    ++q;
                }
            }
            for (int q = lane; q <= npairs; q += 32) rd[q] = q < npairs ? rs[2 * q] : Lp;
            __syncwarp();
            { uint64_t *t = src; src = dst; dst = t; }
            { int *t = rs; rs = rd; rd = t; }
            R = npairs;
        }
        // 3. fp64 reduction of the sorted products (sentinels last), in place at the row head
        int ob = 0;
        int32_t *__restrict__ out_col = chat_col + m0.s;
        float *__restrict__ out_val = chat_val + m0.s;
        for (int p0 = 0; p0 < Lv; p0 += 32) {
            const int p = p0 + lane;
            const bool in = p < Lv;
            const uint64_t x = in ? src[p] : kKvMax;
            const int32_t k = kv_key(x);
            int32_t prev = __shfl_up_sync(kFull, k, 1);
            if (lane == 0) prev = p0 > 0 ? kv_key(src[p0 - 1]) : ~k;
            int32_t next = __shfl_down_sync(kFull, k, 1);
            if (lane == 31) next = p + 1 < Lv ? kv_key(src[p + 1]) : kKeyPad;
            const bool head = in && k != prev;
            const unsigned hm = __ballot_sync(kFull, head);
            const bool dup = in && next == k;
            if (hm == kFull && !__any_sync(kFull, dup)) {
                out_col[ob + lane] = k;
                out_val[ob + lane] = kv_val(x);
                ob += 32;
                continue;
            }
            double acc = (double)kv_val(x);
            if (head && dup)
                for (int q = p + 1; q < Lv; ++q) {
                    const uint64_t y = src[q];
                    if (kv_key(y) != k) break;
                    acc += (double)kv_val(y);
                }
            if (head) {
                const int o = ob + __popc(hm & lt);
                out_col[o] = k;
                out_val[o] = (float)acc;
            }
            ob += __popc(hm);
        }
        if (lane == 0) ccount[m0.i] = ob;
        __syncwarp();
#pragma unroll
        for (int u = 0; u < 2; ++u) { c[u] = cn[u]; f[u] = fn[u]; }
        m0 = m1;
        m1 = m2;
        r += stride;
    }
}

// Load Ĉ[s, s+L) into smem (cp.async), sort, reduce, write the merged row back to Ĉ[s, ...).
template <int NW, int GROUPS, int CAP>
__device__ __forceinline__ int merge_row_in_smem(const Group<NW, GROUPS> &g, unsigned char *slice, int *sc,
                                                 int32_t *__restrict__ chat_col, float *__restrict__ chat_val,
                                                 int64_t s, int L, int Lval, int32_t *__restrict__ out_col,
                                                 float *__restrict__ out_val) {
    constexpr int T = NW * 32;
    int32_t *k0 = (int32_t *)slice;
    float *v0 = (float *)(slice + CAP * 4);
    int32_t *k1 = (int32_t *)(slice + CAP * 8);
    float *v1 = (float *)(slice + CAP * 12);
    int *bA = (int *)(slice + CAP * 16);
    int *bB = bA + SortSmem<CAP>::kBoundsA;
    for (int p = g.gtid; p < L; p += T) {
        cp_async4(k0 + p, chat_col + s + p);
        cp_async4(v0 + p, chat_val + s + p);
    }
    cp_async_wait_all();
    g.sync();
    const int which = natural_merge_sort<NW, GROUPS, CAP>(g, k0, v0, k1, v1, bA, bB, L, sc);
    // sentinel (padding) keys sort last: the first Lval entries are the row's products
    const int U = segmented_reduce_out<NW, GROUPS>(g, which ? k1 : k0, which ? v1 : v0, Lval, out_col, out_val, sc);
    g.sync();
    return U;
}

template <int NW, int GROUPS, int CAP>
__global__ void __launch_bounds__(NW * 32 * GROUPS) k_merge_rows(const int32_t *__restrict__ rows, int64_t nrows,
                                                                const int64_t *__restrict__ rowoff,
                                                                const int64_t *__restrict__ rowwork,
                                                                int32_t *__restrict__ chat_col,
                                                                float *__restrict__ chat_val,
                                                                int64_t *__restrict__ ccount,
                                                                const unsigned *__restrict__ dev_count,
                                                                const int64_t *__restrict__ crowptr,
                                                                int32_t *__restrict__ out_col,
                                                                float *__restrict__ out_val) {
    if (dev_count) nrows = *dev_count;
    extern __shared__ __align__(16) unsigned char smem_raw[];
    __shared__ int sc_all[GROUPS][NW + 1];
    const Group<NW, GROUPS> g;
    unsigned char *slice = smem_raw + (size_t)g.gid * SortSmem<CAP>::kBytes;
    for (int64_t r = (int64_t)blockIdx.x * GROUPS + g.gid; r < nrows; r += (int64_t)gridDim.x * GROUPS) {
        const int i = rows[r];
        const int64_t s = rowoff[i];
        const int L = (int)(rowoff[i + 1] - s);
        const int64_t o = out_col ? crowptr[i] : s;
        const int U = merge_row_in_smem<NW, GROUPS, CAP>(g, slice, sc_all[g.gid], chat_col, chat_val, s, L,
                                                         (int)rowwork[i], (out_col ? out_col : chat_col) + o,
                                                         (out_col ? out_val : chat_val) + o);
        if (g.gtid == 0) ccount[i] = U;
    }
}

// ------------------------------------------------------------------- limited bin ---
// B-Limiting (L463-L477 L, Fig. 7): limited merge blocks take ~200 KB of shared memory each,
// so one is resident per SM (x limit_ctas_per_sm); the grid is persistent and claims rows
// longest-first.  Per row, by size and density:
//   * L <= kLimCap: the whole row is sorted in smem (natural merge sort) and written in place;
//   * dense rows (many products per column of their span): column windows of kLimWindow
//     columns with an fp64 accumulator + touched bits (a counting sort whose bucket
//     accumulation fuses the segment reduction); runs are swept with monotone cursors;
//   * sparse long rows: column windows sized so their products fit kLimCap; each window's
//     sub-runs (found by binary search from the run cursors) are gathered into smem and
//     merge-sorted.
// The merged output of the two windowed paths is staged in the block's global scratch and
// copied to the head of the row's bucket after the whole row has been read.
// (measured: 256 threads / 3584 slots at 2 blocks per SM made C3's long rows 8.6x slower -- bins
// of the coarse partition overflow the smaller sorter and fall back to the window search)
constexpr int kLimBucketCap = 9216;               // rows up to this were merged by the bucket launch
constexpr int64_t kLimSmallStage = 1 << 18;       // per-block scratch (slots) of the 2 / 4 per SM launch
constexpr int cmax3(int a, int b, int c) { return a > b ? (a > c ? a : c) : (b > c ? b : c); }
constexpr int kCoarseLog = 10;
constexpr int kCoarseBins = 1 << kCoarseLog;
// B-Limiting (Fig. 14's "number of blocks per SM"): a limited merge block of NT threads sorts
// column groups of <= NT * EPT products and takes ~1/(1024/NT) of an SM's shared memory, so
// 1024 / NT blocks are resident per SM (options.limit_ctas_per_sm = 1, 2, 4).
template <int NT>
struct LimCfg {
    static constexpr int kThreads = NT;
    static constexpr int kNW = NT / 32;
    static constexpr int kEPT = NT >= 1024 ? 9 : 8;
    static constexpr int kCap = NT * kEPT;                  // 9216 / 4096 / 2048 products
    static constexpr int kWinLog = NT >= 1024 ? 14 : (NT >= 512 ? 13 : 12);
    static constexpr int kWindow = 1 << kWinLog;            // dense-path column window
    static constexpr int kWords = kWindow / 32;             // touched-column bitmap words of a window
    static constexpr int kSortBytes = cmax3(SortSmem<kCap>::kBytes,                  // merge-path fallback
                                            kCap * 16 + (hidx(ceil_pow2(kCap)) + 4) * 4,   // bucket sort
                                            kWindow * 8 + kWords * 4);               // dense window
    static constexpr int kSmem = kSortBytes + (4 * kCoarseBins + 2) * 4;           // + coarse partition tables
    static constexpr int kPerSM = 1024 / NT;
};

struct LimitedArgs {
    const int32_t *rows;          // limited rows, longest first
    int64_t nrows;
    const int64_t *rowoff;
    const int64_t *rowwork;
    const int64_t *run_start;     // [nrows+1]
    const int64_t *run_base;
    const int32_t *run_len;
    int32_t *chat_col;
    float *chat_val;
    int64_t *ccount;
    int32_t *scratch_cursor;      // [grid][max_deg]
    int32_t *scratch_cnt;         // [grid][max_deg]
    int32_t *scratch_col;         // [grid][stage_cap]
    float *scratch_val;
    int64_t max_deg;
    int64_t stage_cap;
    unsigned long long *row_counter;
    int32_t *out_col;             // merged rows go to out_col/out_val + out_off[i] (NULL: in place)
    float *out_val;
    const int64_t *out_off;
    int skip_small;
    unsigned long long *prof;     // NULL, or per-path clock totals [0..10) (tuning)
    int64_t coarse_cap;           // rows up to this many slots take the coarse-partition path
    unsigned long long *lbi;      // NULL, or per-SM busy times (LBI, Eq. (3))
    int32_t *defer_list;          // non-NULL: rows the coarse partition cannot take go here (row list index)
    unsigned *defer_count;
    int dense_div;                // a row is "dense" (fp64 window accumulator) when products * dense_div >= its span
    const int32_t *rlist;         // non-NULL: process only these row list indices (*rlist_count of them)
    const unsigned *rlist_count;
};

__device__ __forceinline__ void smem_add_f64(double *addr, double v) {
    unsigned long long *a = (unsigned long long *)addr;
    unsigned long long old = *a, assumed;
    do {
        assumed = old;
        old = atomicCAS(a, assumed, __double_as_longlong(__longlong_as_double(assumed) + v));
    } while (old != assumed);
}

// number of entries of run [b, b+len) from position cur whose column is < wend (run sorted)
__device__ __forceinline__ int count_below(const int32_t *__restrict__ col, int64_t b, int cur, int len, int32_t wend) {
    int lo = cur, hi = len;     // first p in [cur, len) with col[b+p] >= wend
    int step = 1;               // galloping from the cursor, then binary search
    while (lo + step < hi && col[b + lo + step - 1] < wend) { lo += step; step <<= 1; }
    hi = min(hi, lo + step);
    while (lo < hi) {
        const int mid = (lo + hi) >> 1;
        if (col[b + mid] < wend) lo = mid + 1; else hi = mid;
    }
    return lo - cur;
}

template <int NT>
__global__ void __launch_bounds__(NT, 1024 / NT) k_merge_limited(LimitedArgs g) {
    using C = LimCfg<NT>;
    lbi_start(g.lbi);
    extern __shared__ __align__(16) unsigned char smem_raw[];
    __shared__ int sc[2 * C::kNW + 2];
    __shared__ int64_t row_sm;
    const Group<C::kNW, 1> grp;
    const int lane = lane_id(), w = warp_id();
    int32_t *cursor = g.scratch_cursor + (int64_t)blockIdx.x * g.max_deg;
    int32_t *cnt = g.scratch_cnt + (int64_t)blockIdx.x * g.max_deg;
    int32_t *st_col = g.scratch_col + (int64_t)blockIdx.x * g.stage_cap;
    float *st_val = g.scratch_val + (int64_t)blockIdx.x * g.stage_cap;
    while (true) {
        if (threadIdx.x == 0) row_sm = (int64_t)atomicAdd(g.row_counter, 1ull);
        __syncthreads();
        int64_t r = row_sm;
        __syncthreads();
        if (r >= g.nrows) break;
        if (g.rlist) {
            if (r >= (int64_t)*g.rlist_count) break;
            r = g.rlist[r];
        }
        const int i = g.rows[r];
        const int64_t s = g.rowoff[i];
        const int64_t cap = g.rowoff[i + 1] - s;   // padded bucket length
        const int64_t L = g.rowwork[i];             // products
        const long long t_row = clock64();
        auto rec = [&](int path) {   // options.reserved[1] = 3: per-path row clocks (tuning)
            if (g.prof && threadIdx.x == 0) {
                const unsigned long long dt = (unsigned long long)(clock64() - t_row);
                atomicAdd(g.prof + path, dt);
                atomicAdd(g.prof + 5 + path, 1ull);
                atomicMax(g.prof + 4, dt);
            }
        };
        if (cap <= kLimBucketCap && g.skip_small && g.ccount[i] >= 0) continue;   // merged by the bucket launch
        if (g.defer_list && cap > g.stage_cap) {   // (longer than this launch's per-block scratch)
            if (threadIdx.x == 0) g.defer_list[atomicAdd(g.defer_count, 1u)] = (int32_t)r;
            continue;
        }
        int32_t *const oc = g.out_col ? g.out_col + g.out_off[i] : g.chat_col + s;
        float *const ov = g.out_col ? g.out_val + g.out_off[i] : g.chat_val + s;
        if (cap <= C::kCap) {
            int32_t *dk = (int32_t *)smem_raw;
            float *dv = (float *)(smem_raw + C::kCap * 4);
            int32_t *dk2 = (int32_t *)(smem_raw + C::kCap * 8);
            float *dv2 = (float *)(smem_raw + C::kCap * 12);
            int *hist = (int *)(smem_raw + C::kCap * 16);
            int U = bucket_sort_reduce<C::kNW, 1, C::kEPT, (NT >= 1024 ? SPG_LIM_LS : 0), SPG_LIM_UNR2>(grp, g.chat_col + s, g.chat_val + s, (int)cap, dk, dv, dk2,
                                                            dv2, hist, oc, ov, sc);
            if (U < 0)
                U = merge_row_in_smem<C::kNW, 1, C::kCap>(grp, smem_raw, sc, g.chat_col, g.chat_val, s, (int)cap, (int)L,
                                                          oc, ov);
            if (threadIdx.x == 0) g.ccount[i] = U;
            __syncthreads();
            rec(0);
            continue;
        }
        const int64_t rs = g.run_start[r];
        const int R = (int)(g.run_start[r + 1] - rs);
        const int64_t *rbase = g.run_base + rs;
        const int32_t *rlen = g.run_len + rs;
        int32_t mn = kKeyPad, mx = 0;
        for (int q = threadIdx.x; q < R; q += C::kThreads) {
            const int64_t b = rbase[q];
            mn = min(mn, g.chat_col[b]);
            mx = max(mx, g.chat_col[b + rlen[q] - 1]);
            cursor[q] = 0;
        }
        mn = grp.reduce_min(mn, sc);
        mx = grp.reduce_max(mx, sc);
        const int64_t span = (int64_t)mx - mn + 1;
        const int64_t nwin_dense = (span + C::kWindow - 1) / C::kWindow;
        const bool dense = L * g.dense_div >= span && (int64_t)R * nwin_dense <= 2 * L;
        int64_t nout = 0;
        const int64_t nwin_pow = (span + C::kWindow - 1) >> C::kWinLog;
        if (dense && cap <= g.stage_cap && nwin_pow <= kCoarseBins) {
            // dense row, streamed: (1) histogram of the row's column windows (2^C::kWinLog columns),
            // (2) scatter into the block's scratch grouped by window, (3) per window, coalesced
            // sweep of its products into the fp64 shared accumulator + touched bits, extracted in
            // column order straight to the row's output (the row now lives in scratch).  Every
            // load is independent (the per-run cursor walk below is one dependent load per run
            // per window: C3's hub rows, 38K runs x 104 windows, took 250 ms in one block).
            const int nwin = (int)nwin_pow;
            int *fh = (int *)(smem_raw + C::kSortBytes);       // [kCoarseBins] counts -> starts
            int *wst = fh + kCoarseBins;                        // [kCoarseBins + 1]
            int *wcur = wst + kCoarseBins + 1;                  // [kCoarseBins]
            int32_t *sc_col = g.scratch_col + (int64_t)blockIdx.x * g.stage_cap;
            float *sc_val = g.scratch_val + (int64_t)blockIdx.x * g.stage_cap;
            for (int t = threadIdx.x; t < kCoarseBins; t += C::kThreads) fh[t] = 0;
            __syncthreads();
            for (int64_t p = threadIdx.x; p < (cap >> 2); p += C::kThreads) {
                const int4 c4 = *reinterpret_cast<const int4 *>(g.chat_col + s + 4 * p);
                const int32_t cc[4] = {c4.x, c4.y, c4.z, c4.w};
#pragma unroll
                for (int u = 0; u < 4; ++u) {
                    const int wid = cc[u] == kKeyPad ? -1 - lane_id() : (cc[u] - mn) >> C::kWinLog;
                    const unsigned peers = __match_any_sync(__activemask(), wid);
                    if (wid >= 0 && lane_id() == __ffs(peers) - 1) atomicAdd(&fh[wid], __popc(peers));
                }
            }
            __syncthreads();
            {
                constexpr int BPT = kCoarseBins / C::kThreads;
                int c[BPT], cnt = 0;
#pragma unroll
                for (int u = 0; u < BPT; ++u) { c[u] = fh[threadIdx.x * BPT + u]; cnt += c[u]; }
                int tot;
                int ex = grp.excl_sum(cnt, sc, &tot);
#pragma unroll
                for (int u = 0; u < BPT; ++u) {
                    wst[threadIdx.x * BPT + u] = ex;
                    wcur[threadIdx.x * BPT + u] = ex;
                    ex += c[u];
                }
                if (threadIdx.x == 0) wst[kCoarseBins] = tot;
            }
            __syncthreads();
            for (int64_t p = threadIdx.x; p < (cap >> 2); p += C::kThreads) {
                const int4 c4 = *reinterpret_cast<const int4 *>(g.chat_col + s + 4 * p);
                const float4 v4 = *reinterpret_cast<const float4 *>(g.chat_val + s + 4 * p);
                const int32_t cc[4] = {c4.x, c4.y, c4.z, c4.w};
                const float vv[4] = {v4.x, v4.y, v4.z, v4.w};
#pragma unroll
                for (int u = 0; u < 4; ++u) {     // warp-aggregated cursor bumps per window
                    const int wid = cc[u] == kKeyPad ? -1 - lane_id() : (cc[u] - mn) >> C::kWinLog;
                    const unsigned peers = __match_any_sync(__activemask(), wid);
                    if (wid >= 0) {
                        const int leader = __ffs(peers) - 1;
                        int q0 = 0;
                        if (lane_id() == leader) q0 = atomicAdd(&wcur[wid], __popc(peers));
                        q0 = __shfl_sync(peers, q0, leader);
                        const int q = q0 + __popc(peers & lanemask_lt());
                        sc_col[q] = cc[u];
                        sc_val[q] = vv[u];
                    }
                }
            }
            double *acc = (double *)smem_raw;
            uint32_t *bits = (uint32_t *)(smem_raw + C::kWindow * 8);
            for (int t = threadIdx.x; t < C::kWindow; t += C::kThreads) acc[t] = 0.0;
            for (int t = threadIdx.x; t < C::kWindow / 32; t += C::kThreads) bits[t] = 0u;
            __syncthreads();
            for (int wi = 0; wi < nwin; ++wi) {
                const int q0 = wst[wi], q1 = wst[wi + 1];
                if (q0 == q1) continue;
                const int32_t wbase = mn + (wi << C::kWinLog);
                for (int q = q0 + threadIdx.x; q < q1; q += C::kThreads) {
                    const int x = sc_col[q] - wbase;
                    smem_add_f64(acc + x, (double)sc_val[q]);
                    atomicOr(bits + (x >> 5), 1u << (x & 31));
                }
                __syncthreads();
                constexpr int WPT = C::kWords >= C::kThreads ? C::kWords / C::kThreads : 1;
                const bool own = threadIdx.x * WPT < C::kWords;   // threads past the bitmap: no words
                int cntw = 0;
                uint32_t word[WPT];
#pragma unroll
                for (int u = 0; u < WPT; ++u) {
                    word[u] = own ? bits[threadIdx.x * WPT + u] : 0u;
                    cntw += __popc(word[u]);
                }
                int tot;
                int64_t pos = nout + grp.excl_sum(cntw, sc, &tot);
#pragma unroll
                for (int u = 0; u < WPT; ++u) {
                    uint32_t m = word[u];
                    while (m) {
                        const int bpos = __ffs(m) - 1;
                        m &= m - 1;
                        const int x = (threadIdx.x * WPT + u) * 32 + bpos;
                        oc[pos] = wbase + x;
                        ov[pos] = (float)acc[x];
                        acc[x] = 0.0;
                        ++pos;
                    }
                    if (own) bits[threadIdx.x * WPT + u] = 0u;
                }
                nout += tot;
                __syncthreads();
            }
            if (threadIdx.x == 0) g.ccount[i] = nout;
            __syncthreads();
            rec(2);
            continue;
        }
        if (dense) {
            double *acc = (double *)smem_raw;
            uint32_t *bits = (uint32_t *)(smem_raw + C::kWindow * 8);
            for (int t = threadIdx.x; t < C::kWindow; t += C::kThreads) acc[t] = 0.0;
            for (int t = threadIdx.x; t < C::kWindow / 32; t += C::kThreads) bits[t] = 0u;
            __syncthreads();
            for (int64_t w0 = mn; w0 <= mx; w0 += C::kWindow) {
                const int32_t wend = (int32_t)min((int64_t)mx + 1, w0 + C::kWindow);
                // warp per run, 32 products per step: a run contributes L / (R * #windows) < 2
                // products to a window on average, so a wider probe mostly loads entries of later
                // windows (measured: 4 vectors per lane made C3's densest rows 4x slower)
                for (int q = w; q < R; q += C::kNW) {
                    const int64_t b = rbase[q];
                    const int len = rlen[q];
                    int cur = cursor[q];
                    while (cur < len) {
                        const int p = cur + lane;
                        const int32_t c = p < len ? g.chat_col[b + p] : kKeyPad;
                        const bool in = c < wend;
                        if (in) {
                            const int x = c - (int32_t)w0;
                            smem_add_f64(acc + x, (double)g.chat_val[b + p]);
                            atomicOr(bits + (x >> 5), 1u << (x & 31));
                        }
                        const int taken = __popc(__ballot_sync(kFull, in));
                        cur += taken;
                        if (taken < 32) break;
                    }
                    if (lane == 0) cursor[q] = cur;
                }
                __syncthreads();
                constexpr int WPT = C::kWords >= C::kThreads ? C::kWords / C::kThreads : 1;
                const bool own = threadIdx.x * WPT < C::kWords;   // threads past the bitmap: no words
                int cntw = 0;
                uint32_t word[WPT];
#pragma unroll
                for (int u = 0; u < WPT; ++u) {
                    word[u] = own ? bits[threadIdx.x * WPT + u] : 0u;
                    cntw += __popc(word[u]);
                }
                int tot;
                int64_t pos = nout + grp.excl_sum(cntw, sc, &tot);
#pragma unroll
                for (int u = 0; u < WPT; ++u) {
                    uint32_t m = word[u];
                    while (m) {
                        const int bpos = __ffs(m) - 1;
                        m &= m - 1;
                        const int x = (threadIdx.x * WPT + u) * 32 + bpos;
                        st_col[pos] = (int32_t)w0 + x;
                        st_val[pos] = (float)acc[x];
                        acc[x] = 0.0;
                        ++pos;
                    }
                    if (own) bits[threadIdx.x * WPT + u] = 0u;
                }
                nout += tot;
                __syncthreads();
            }
        } else {
            bool done_coarse = false;
            if (cap <= g.coarse_cap) {
                long long t_c = clock64();
                auto sub = [&](int slot) {   // coarse-path sub-phase clocks (tuning, reserved[1] = 3)
                    if (g.prof && threadIdx.x == 0) {
                        const long long t = clock64();
                        atomicAdd(g.prof + slot, (unsigned long long)(t - t_c));
                        t_c = t;
                    }
                };
                // sparse long row: coarse column partition through global scratch (two coalesced passes)
                //  1. histogram over kCoarseBins column ranges; greedy groups of <= C::kCap entries
                //  2. scatter the row into the block's scratch, grouped by column range
                //  3. per group (ascending): smem bucket sort (merge-path fallback), merged entries
                //     appended at the head of the row's bucket -- the row now lives in scratch
                int *fh = (int *)(smem_raw + C::kSortBytes);      // [kCoarseBins] counts -> group id
                int *gstart = fh + kCoarseBins;                    // [kCoarseBins + 1]
                int *gcur = gstart + kCoarseBins + 1;              // [kCoarseBins]
                int *gbin = gcur + kCoarseBins;                    // [kCoarseBins + 1] first bin of each group
                __shared__ int s_ngroups, s_bad;
                const uint32_t span32 = (uint32_t)(mx - mn);
                const int bits = span32 ? 32 - __clz(span32) : 0;
                const int shc = max(0, bits - kCoarseLog);
                for (int t = threadIdx.x; t < kCoarseBins; t += C::kThreads) fh[t] = 0;
                __syncthreads();
                for (int64_t p = threadIdx.x; p < (cap >> 2); p += C::kThreads) {
                    const int4 c4 = *reinterpret_cast<const int4 *>(g.chat_col + s + 4 * p);
                    if (c4.x != kKeyPad) atomicAdd(&fh[(c4.x - mn) >> shc], 1);
                    if (c4.y != kKeyPad) atomicAdd(&fh[(c4.y - mn) >> shc], 1);
                    if (c4.z != kKeyPad) atomicAdd(&fh[(c4.z - mn) >> shc], 1);
                    if (c4.w != kKeyPad) atomicAdd(&fh[(c4.w - mn) >> shc], 1);
                }
                __syncthreads();
                {   // grouping of consecutive bins: group(b) = floor(prefix(b) / (C::kCap/2)); with no bin
                    // above C::kCap/2 a group holds < C::kCap products.  Bins per thread: 2 (1024 / 512).
                    constexpr int BPT = kCoarseBins / C::kThreads;
                    int c[BPT], cnt = 0, mxb = 0;
#pragma unroll
                    for (int u = 0; u < BPT; ++u) {
                        c[u] = fh[threadIdx.x * BPT + u];
                        cnt += c[u];
                        mxb = max(mxb, c[u]);
                    }
                    int tot;
                    int ex = grp.excl_sum(cnt, sc, &tot);
                    mxb = grp.reduce_max(mxb, sc);
                    // groups < T + max bin <= C::kCap: 3/4 of the sorter when no bin exceeds 1/4 of it
                    // (fewer, fuller sorts: C3 182 -> 159 ms; 7/8: same speed), else 1/2, so rows
                    // with one heavy column range still take this path (C5: 3/4 alone sent them to
                    // the window path, limited merge 86 -> 115 ms)
                    const int T = SPG_LIM_T78 && mxb <= C::kCap / 8 ? C::kCap * 7 / 8
                                                                     : (mxb <= C::kCap / 4 ? C::kCap * 3 / 4 : C::kCap / 2);
#pragma unroll
                    for (int u = 0; u < BPT; ++u) {
                        fh[threadIdx.x * BPT + u] = ex / T;     // group id of the bin
                        ex += c[u];
                    }
                    const int ng = (tot + T - 1) / T;
                    // (group ids are prefix / T: more of them than table slots when the row holds more than
                    // kCoarseBins * T products -- the smaller sorters of 2 / 4 blocks per SM: not this path)
                    const bool over = ng > kCoarseBins;
                    // group start = first prefix value >= gi*T, i.e. prefix of the first bin of group gi
                    if (!over)
                        for (int gi = threadIdx.x; gi <= ng; gi += C::kThreads) { gstart[gi] = 0x7fffffff; gbin[gi] = 0x7fffffff; }
                    __syncthreads();
                    int pre = ex - cnt;
                    if (!over) {
#pragma unroll
                        for (int u = 0; u < BPT; ++u) {
                            atomicMin(&gstart[pre / T], pre);
                            atomicMin(&gbin[pre / T], threadIdx.x * BPT + u);
                            pre += c[u];
                        }
                    }
                    if (threadIdx.x == 0) {
                        s_ngroups = ng;
                        s_bad = over || mxb > C::kCap - T;
                        if (!over) {
                            gstart[ng] = tot;
                            gbin[ng] = kCoarseBins;
                        }
                    }
                    __syncthreads();
                    // groups with no bin starting inside them cannot exist (bins are contiguous), but
                    // guard: an untouched start inherits the next group's start (empty group)
                    if (threadIdx.x == 0 && !over)
                        for (int gi = ng - 1; gi >= 0; --gi)
                            if (gstart[gi] == 0x7fffffff) { gstart[gi] = gstart[gi + 1]; gbin[gi] = gbin[gi + 1]; }
                }
                __syncthreads();
                sub(10);   // min/max, histogram, grouping
                if (!s_bad) {   // (a single column range holding > C::kCap products: window path)
                    const int ng = s_ngroups;
                    int32_t *sc_col = g.scratch_col + (int64_t)blockIdx.x * g.stage_cap;
                    float *sc_val = g.scratch_val + (int64_t)blockIdx.x * g.stage_cap;
                    for (int t = threadIdx.x; t < ng; t += C::kThreads) gcur[t] = gstart[t];
                    __syncthreads();
                    for (int64_t p = threadIdx.x; p < (cap >> 2); p += C::kThreads) {
                        const int4 c4 = *reinterpret_cast<const int4 *>(g.chat_col + s + 4 * p);
                        const float4 v4 = *reinterpret_cast<const float4 *>(g.chat_val + s + 4 * p);
                        const int32_t cc[4] = {c4.x, c4.y, c4.z, c4.w};
                        const float vv[4] = {v4.x, v4.y, v4.z, v4.w};
#pragma unroll
                        for (int u = 0; u < 4; ++u) {     // warp-aggregated cursor bumps per group
                            const int gid = cc[u] == kKeyPad ? -1 - lane_id() : fh[(cc[u] - mn) >> shc];
#if SPG_SCATTER_BALLOT
                            {   // the warp's groups span a few ids: one ballot per id instead of a match
                                const unsigned act = __activemask();
                                const int glo = __reduce_min_sync(act, gid >= 0 ? gid : 0x7fffffff);
                                const int ghi = __reduce_max_sync(act, gid);
                                if (ghi - glo < 4) {
                                    for (int gq = glo; gq <= ghi; ++gq) {
                                        const unsigned m = __ballot_sync(act, gid == gq);
                                        if (!m) continue;
                                        const int leader = __ffs(m) - 1;
                                        int q0 = 0;
                                        if (lane_id() == leader) q0 = atomicAdd(&gcur[gq], __popc(m));
                                        q0 = __shfl_sync(act, q0, leader);
                                        if (gid == gq) {
                                            const int q = q0 + __popc(m & lanemask_lt());
                                            sc_col[q] = cc[u];
                                            sc_val[q] = vv[u];
                                        }
                                    }
                                    continue;
                                }
                            }
#endif
                            const unsigned peers = __match_any_sync(__activemask(), gid);
                            if (gid >= 0) {
                                const int leader = __ffs(peers) - 1;
                                int q0 = 0;
                                if (lane_id() == leader) q0 = atomicAdd(&gcur[gid], __popc(peers));
                                q0 = __shfl_sync(peers, q0, leader);
                                const int q = q0 + __popc(peers & lanemask_lt());
                                sc_col[q] = cc[u];
                                sc_val[q] = vv[u];
                            }
                        }
                    }
                    __syncthreads();
                    sub(11);   // scatter into scratch
#if SPG_LIM_GPIPE
                    // software-pipelined group sorts: group gi + 1's products are loaded from the scratch
                    // (L2) into registers while group gi sorts
                    int32_t key[C::kEPT];
                    float val[C::kEPT];
                    bsr_load<C::kNW, 1, C::kEPT>(grp, sc_col + gstart[0], sc_val + gstart[0], ng > 0 ? gstart[1] - gstart[0] : 0,
                                                 key, val);
#endif
                    for (int gi = 0; gi < ng; ++gi) {
                        const int g0 = gstart[gi], n = gstart[gi + 1] - g0;
#if SPG_LIM_GPIPE
                        int32_t kn[C::kEPT];
                        float vn[C::kEPT];
                        {
                            const int g1 = gi + 1 < ng ? gstart[gi + 1] : 0;
                            const int n1 = gi + 1 < ng ? gstart[gi + 2] - g1 : 0;
                            bsr_load<C::kNW, 1, C::kEPT>(grp, sc_col + g1, sc_val + g1, n1, kn, vn);
                        }
#endif
                        if (n > 0) {
                        // the group's column range from its coarse bins (no min / max reduction)
                        const int32_t gmn = (int32_t)((int64_t)mn + ((int64_t)gbin[gi] << shc));
                        const int32_t gmx = (int32_t)min((int64_t)mx, (int64_t)mn + ((int64_t)gbin[gi + 1] << shc) - 1);
#if SPG_LIM_GPIPE
                        int U = bucket_sort_reduce_regs<C::kNW, 1, C::kEPT, 0, SPG_LIM_UNR2>(
                            grp, key, val, n, (int32_t *)smem_raw, (float *)(smem_raw + C::kCap * 4),
                            (int32_t *)(smem_raw + C::kCap * 8), (float *)(smem_raw + C::kCap * 12),
                            (int *)(smem_raw + C::kCap * 16), oc + nout, ov + nout, sc, gmn, gmx);
#else
                        int U = bucket_sort_reduce<C::kNW, 1, C::kEPT, (NT >= 1024 ? SPG_LIM_LS : 0), SPG_LIM_UNR2>(
                            grp, sc_col + g0, sc_val + g0, n, (int32_t *)smem_raw, (float *)(smem_raw + C::kCap * 4),
                            (int32_t *)(smem_raw + C::kCap * 8), (float *)(smem_raw + C::kCap * 12),
                            (int *)(smem_raw + C::kCap * 16), oc + nout, ov + nout, sc, gmn, gmx);
#endif
                        if (U < 0)
                            U = merge_row_in_smem<C::kNW, 1, C::kCap>(grp, smem_raw, sc, sc_col, sc_val, g0, n, n,
                                                                      oc + nout, ov + nout);
                        nout += U;
                        __syncthreads();
                        }
#if SPG_LIM_GPIPE
#pragma unroll
                        for (int e = 0; e < C::kEPT; ++e) { key[e] = kn[e]; val[e] = vn[e]; }
#endif
                    }
                    if (threadIdx.x == 0) g.ccount[i] = nout;
                    __syncthreads();
                    sub(12);   // group sorts
                    if (g.prof && threadIdx.x == 0) atomicAdd(g.prof + 13, (unsigned long long)ng);
                    done_coarse = true;
                }
                __syncthreads();
            }
            if (done_coarse) { rec(1); continue; }
            if (g.defer_list) {   // (a column range too heavy for this block's sorter: the 1-per-SM launch)
                if (threadIdx.x == 0) g.defer_list[atomicAdd(g.defer_count, 1u)] = (int32_t)r;
                continue;
            }
            // sparse: windows whose products fit the smem sorter
            int32_t *k0 = (int32_t *)smem_raw;
            float *v0 = (float *)(smem_raw + C::kCap * 4);
            int64_t remaining = L;
            int64_t w0 = mn;
            while (w0 <= mx) {
                int64_t width = max((int64_t)1, (int64_t)((double)(mx + 1 - w0) * (C::kCap / 2) / (double)max(remaining, (int64_t)1)));
                int total = 0;
                int32_t wend = 0;
                int32_t head = kKeyPad;
                while (true) {
                    wend = (int32_t)min((int64_t)mx + 1, w0 + width);
                    int part = 0;
                    int32_t hmin = kKeyPad;
                    for (int q = threadIdx.x; q < R; q += C::kThreads) {
                        const int64_t b = rbase[q];
                        const int cur = cursor[q], len = rlen[q];
                        if (cur < len) hmin = min(hmin, g.chat_col[b + cur]);
                        const int c = count_below(g.chat_col, b, cur, len, wend);
                        cnt[q] = c;
                        part += c;
                    }
                    int tot;
                    grp.excl_sum(part, sc, &tot);
                    total = tot;
                    head = grp.reduce_min(hmin, sc);
                    if (total <= C::kCap || width == 1) break;
                    width = max((int64_t)1, width / 2);
                }
                if (total == 0) {              // empty window: jump to the next product's column
                    w0 = max((int64_t)wend, (int64_t)head);
                    continue;
                }
                if (total > C::kCap) {         // one column (w0) present in > C::kCap runs
                    double part = 0.0;
                    for (int q = threadIdx.x; q < R; q += C::kThreads) {
                        if (cnt[q] > 0) {
                            part += (double)g.chat_val[rbase[q] + cursor[q]];
                            cursor[q] += 1;
                        }
                    }
                    part = warp_sum(part);
                    __shared__ double dred[C::kNW];
                    if (lane == 0) dred[w] = part;
                    __syncthreads();
                    if (threadIdx.x == 0) {
                        double t = 0.0;
                        for (int q = 0; q < C::kNW; ++q) t += dred[q];
                        st_col[nout] = (int32_t)w0;
                        st_val[nout] = (float)t;
                    }
                    __syncthreads();
                    nout += 1;
                    remaining -= total;
                    w0 = wend;
                    continue;
                }
                // exclusive scan of cnt[0..R) into offsets (cnt[R] = total), then warp-per-run gather
                int base_off = 0;
                for (int q0 = 0; q0 < R; q0 += C::kThreads) {
                    const int q = q0 + threadIdx.x;
                    const int c = q < R ? cnt[q] : 0;
                    int tot;
                    const int ex = grp.excl_sum(c, sc, &tot);
                    if (q < R) cnt[q] = base_off + ex;
                    base_off += tot;
                }
                if (threadIdx.x == 0) cnt[R] = base_off;
                __syncthreads();
                for (int q = w; q < R; q += C::kNW) {
                    const int off = cnt[q], c = cnt[q + 1] - off;
                    if (c == 0) continue;
                    const int64_t b = rbase[q] + cursor[q];
                    for (int t = lane; t < c; t += 32) {
                        cp_async4(k0 + off + t, g.chat_col + b + t);
                        cp_async4(v0 + off + t, g.chat_val + b + t);
                    }
                    if (lane == 0) cursor[q] += c;
                }
                cp_async_wait_all();
                __syncthreads();
                int U = bucket_sort_reduce<C::kNW, 1, C::kEPT, (NT >= 1024 ? SPG_LIM_LS : 0), SPG_LIM_UNR2>(grp, k0, v0, total, k0, v0,
                                                                (int32_t *)(smem_raw + C::kCap * 8),
                                                                (float *)(smem_raw + C::kCap * 12),
                                                                (int *)(smem_raw + C::kCap * 16), st_col + nout,
                                                                st_val + nout, sc);
                if (U < 0) {
                    int32_t *k1 = (int32_t *)(smem_raw + C::kCap * 8);
                    float *v1 = (float *)(smem_raw + C::kCap * 12);
                    int *bA = (int *)(smem_raw + C::kCap * 16);
                    int *bB = bA + SortSmem<C::kCap>::kBoundsA;
                    const int which = natural_merge_sort<C::kNW, 1, C::kCap>(grp, k0, v0, k1, v1, bA, bB, total, sc);
                    U = segmented_reduce_out<C::kNW, 1>(grp, which ? k1 : k0, which ? v1 : v0, total,
                                                        st_col + nout, st_val + nout, sc);
                }
                __syncthreads();
                nout += U;
                remaining -= total;
                w0 = wend;
            }
        }
        // copy the merged row to its output (side buffer, or the head of its Ĉ bucket)
        for (int64_t p = threadIdx.x; p < nout; p += C::kThreads) {
            oc[p] = st_col[p];
            ov[p] = st_val[p];
        }
        if (threadIdx.x == 0) g.ccount[i] = nout;
        __syncthreads();
        rec(dense ? 2 : 3);
    }
    lbi_end(g.lbi);
}

// Single-run rows: already sorted and duplicate-free; merged length = bucket length.
__global__ void k_merge_pass(const int32_t *__restrict__ rows, int64_t nrows, const int64_t *__restrict__ rowwork,
                             int64_t *__restrict__ ccount) {
    for (int64_t q = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; q < nrows; q += (int64_t)gridDim.x * blockDim.x) {
        const int i = rows[q];
        ccount[i] = rowwork[i];   // the run's sentinel padding trails its products
    }
}

// ------------------------------------------------------------------ CSR compaction ---
// Row i's merged entries sit at Ĉ[rowoff[i] ..) and move to C[crowptr[i] ..).  One warp per
// row (4 loads in flight per lane); rows longer than kCompactWarpMax get a CTA each.
constexpr int kCompactWarpMax = 8192;
constexpr int kCompactLongThreads = 512;

// Realign 4-wide vectors for an output shifted by sh (dst mod 4): the aligned output vector of
// lane m holds source elements [4m - sh, 4m - sh + 4): the last sh of the previous vector and
// the first 4 - sh of this lane's.  `prev` = the previous lane's vector (lane 0: carried).
template <typename V>
__device__ __forceinline__ V realign4(const V &cur, const V &prev, int sh) {
    V o;
    switch (sh) {
        case 0: o = cur; break;
        case 1: o.x = prev.w; o.y = cur.x; o.z = cur.y; o.w = cur.z; break;
        case 2: o.x = prev.z; o.y = prev.w; o.z = cur.x; o.w = cur.y; break;
        default: o.x = prev.y; o.y = prev.z; o.z = prev.w; o.w = cur.x; break;
    }
    return o;
}

template <typename V>
__device__ __forceinline__ V shfl_up_vec(const V &v, const V &carry) {
    V p;
    p.x = __shfl_up_sync(kFull, v.x, 1);
    p.y = __shfl_up_sync(kFull, v.y, 1);
    p.z = __shfl_up_sync(kFull, v.z, 1);
    p.w = __shfl_up_sync(kFull, v.w, 1);
    if (lane_id() == 0) p = carry;
    return p;
}

__global__ void __launch_bounds__(256) k_compact_rows(const int32_t *__restrict__ list,
                                                      const int64_t *__restrict__ crowptr, int64_t M,
                                                      const int64_t *__restrict__ rowoff,
                                                      const int32_t *__restrict__ chat_col,
                                                      const float *__restrict__ chat_val,
                                                      int32_t *__restrict__ out_col, float *__restrict__ out_val) {
    const int lane = lane_id();
    for (int64_t q = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; q < M;
         q += ((int64_t)gridDim.x * blockDim.x) >> 5) {
        const int64_t i = list ? list[q] : q;       // M = list length when a list is given
        const int64_t dst = crowptr[i];
        const int64_t cnt = crowptr[i + 1] - dst;
        if (cnt == 0 || cnt > kCompactWarpMax) continue;
        const int64_t src = rowoff[i];               // 16-byte aligned (padded runs)
        const int sh = (int)(dst & 3);
        const int64_t dst_a = dst - sh;              // aligned output base
        // aligned output vector m covers output slots [4m - sh, 4m - sh + 4) of the row
        const int64_t nvec = (cnt + sh + 3) >> 2;
        int4 carry_c = make_int4(0, 0, 0, 0);
        float4 carry_v = make_float4(0.f, 0.f, 0.f, 0.f);
        auto emit = [&](int64_t m, const int4 &c, const float4 &v) {
            const int4 oc = realign4(c, shfl_up_vec(c, carry_c), sh);
            const float4 ov = realign4(v, shfl_up_vec(v, carry_v), sh);
            carry_c.x = __shfl_sync(kFull, c.x, 31); carry_c.y = __shfl_sync(kFull, c.y, 31);
            carry_c.z = __shfl_sync(kFull, c.z, 31); carry_c.w = __shfl_sync(kFull, c.w, 31);
            carry_v.x = __shfl_sync(kFull, v.x, 31); carry_v.y = __shfl_sync(kFull, v.y, 31);
            carry_v.z = __shfl_sync(kFull, v.z, 31); carry_v.w = __shfl_sync(kFull, v.w, 31);
            if (m < nvec) {
                const int64_t j0 = 4 * m - sh;       // row slot of the vector's first element
                if (j0 >= 0 && j0 + 4 <= cnt) {
                    __stcs(reinterpret_cast<int4 *>(out_col + dst_a + 4 * m), oc);
                    __stcs(reinterpret_cast<float4 *>(out_val + dst_a + 4 * m), ov);
                } else {                              // ragged head / tail of the row
                    const int32_t cc[4] = {oc.x, oc.y, oc.z, oc.w};
                    const float vv[4] = {ov.x, ov.y, ov.z, ov.w};
#pragma unroll
                    for (int u = 0; u < 4; ++u)
                        if (j0 + u >= 0 && j0 + u < cnt) {
                            out_col[dst_a + 4 * m + u] = cc[u];
                            out_val[dst_a + 4 * m + u] = vv[u];
                        }
                }
            }
        };
        for (int64_t m0 = 0; m0 < nvec; m0 += 64) {   // two vectors in flight per lane
            int4 c[2];
            float4 v[2];
#pragma unroll
            for (int u = 0; u < 2; ++u) {
                const int64_t m = m0 + 32 * u + lane;
                c[u] = make_int4(0, 0, 0, 0);
                v[u] = make_float4(0.f, 0.f, 0.f, 0.f);
                if (4 * m < cnt) {
                    c[u] = __ldcs(reinterpret_cast<const int4 *>(chat_col + src + 4 * m));
                    v[u] = __ldcs(reinterpret_cast<const float4 *>(chat_val + src + 4 * m));
                }
            }
            emit(m0 + lane, c[0], v[0]);
            if (m0 + 32 < nvec) emit(m0 + 32 + lane, c[1], v[1]);
        }
    }
}

__global__ void __launch_bounds__(kCompactLongThreads) k_compact_long(const int32_t *__restrict__ rows, int64_t nrows,
                                                                      const int64_t *__restrict__ crowptr,
                                                                      const int64_t *__restrict__ rowoff,
                                                                      const int32_t *__restrict__ chat_col,
                                                                      const float *__restrict__ chat_val,
                                                                      int32_t *__restrict__ out_col,
                                                                      float *__restrict__ out_val) {
    for (int64_t r = blockIdx.x; r < nrows; r += gridDim.x) {
        const int i = rows[r];
        const int64_t dst = crowptr[i];
        const int64_t cnt = crowptr[i + 1] - dst;
        if (cnt <= kCompactWarpMax) continue;
        const int64_t src = rowoff[i];
        for (int64_t p0 = 0; p0 < cnt; p0 += 4 * kCompactLongThreads) {
            int32_t c[4];
            float v[4];
#pragma unroll
            for (int q = 0; q < 4; ++q) {
                const int64_t p = p0 + q * kCompactLongThreads + threadIdx.x;
                c[q] = p < cnt ? chat_col[src + p] : 0;
                v[q] = p < cnt ? chat_val[src + p] : 0.f;
            }
#pragma unroll
            for (int q = 0; q < 4; ++q) {
                const int64_t p = p0 + q * kCompactLongThreads + threadIdx.x;
                if (p < cnt) {
                    out_col[dst + p] = c[q];
                    out_val[dst + p] = v[q];
                }
            }
        }
    }
}

// Load-balanced compaction: the output is cut into chunks of kCmpChunk entries (a chunk may
// hold part of one long row or many short rows); chunk_r0[c] = row of the chunk's first entry.
// A thread writes aligned 16-byte output vectors; each of its 4 entries is read from its row's
// bucket head (src = rowoff[r] + (q - crowptr[r]); 4 scalar loads, coalesced across the warp).
// Every row length gets the same per-entry cost (C3's 60K-entry rows made the warp / CTA per
// row copy 2.4 TB/s).
#ifndef SPG_CMP_CHUNK
#define SPG_CMP_CHUNK 8192
#endif
constexpr int kCmpChunk = SPG_CMP_CHUNK;
#ifndef SPG_CMP_THREADS
#define SPG_CMP_THREADS 256
#endif
constexpr int kCmpThreads = SPG_CMP_THREADS;

__global__ void k_chunk_first_row(const int64_t *__restrict__ crowptr, int64_t M, int64_t nnz, int64_t nchunks,
                                  int32_t *__restrict__ chunk_r0) {
    for (int64_t c = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; c <= nchunks; c += (int64_t)gridDim.x * blockDim.x) {
        const int64_t q = min(c * (int64_t)kCmpChunk, nnz - 1);
        int64_t lo = 0, hi = M;               // last row r with crowptr[r] <= q (a non-empty row)
        while (hi - lo > 1) {
            const int64_t mid = (lo + hi) >> 1;
            if (crowptr[mid] <= q) lo = mid; else hi = mid;
        }
        chunk_r0[c] = (int32_t)lo;
    }
}

__global__ void __launch_bounds__(kCmpThreads) k_compact_flat(const int64_t *__restrict__ crowptr,
                                                               const int64_t *__restrict__ rowoff,
                                                               const int32_t *__restrict__ chunk_r0, int64_t nnz,
                                                               int64_t nchunks, const int32_t *__restrict__ chat_col,
                                                               const float *__restrict__ chat_val,
                                                               int32_t *__restrict__ out_col,
                                                               float *__restrict__ out_val) {
    for (int64_t c = blockIdx.x; c < nchunks; c += gridDim.x) {
        const int64_t q0 = c * (int64_t)kCmpChunk, q1 = min(nnz, q0 + kCmpChunk);
        const int r0 = chunk_r0[c], r1 = chunk_r0[c + 1];
        int rc = r0;                                   // this thread's row cursor (monotone)
        int64_t cs = __ldg(crowptr + rc), ce = __ldg(crowptr + rc + 1), ro = __ldg(rowoff + rc);
        auto seek = [&](int64_t q) {                   // row of entry q (q >= cs): cached bounds
            if (q < ce) return;
            int lo = rc + 1, hi = r1 + 1;              // last row in (rc, r1] with crowptr <= q
            while (hi - lo > 1) {
                const int mid = (lo + hi) >> 1;
                if (__ldg(crowptr + mid) <= q) lo = mid; else hi = mid;
            }
            rc = lo;
            cs = __ldg(crowptr + rc);
            ce = __ldg(crowptr + rc + 1);
            ro = __ldg(rowoff + rc);
        };
        for (int64_t qv = q0 + 4 * threadIdx.x; qv < q1; qv += 4 * kCmpThreads) {
            int32_t cc[4];
            float vv[4];
            seek(qv);
            if (qv + 4 <= q1 && ce >= qv + 4) {
                // the 4 entries are consecutive in one row: two aligned vectors + realign
                const int64_t src = ro + (qv - cs);
                const int sh = (int)(src & 3);
                const int64_t a = src - sh;
                // (default caching: the second vector is the next lane's first -- an L1 hit)
                const int4 c0 = *reinterpret_cast<const int4 *>(chat_col + a);
                const float4 v0 = *reinterpret_cast<const float4 *>(chat_val + a);
                int4 oc = c0;
                float4 ov = v0;
                if (sh) {
                    const int4 c1 = *reinterpret_cast<const int4 *>(chat_col + a + 4);
                    const float4 v1 = *reinterpret_cast<const float4 *>(chat_val + a + 4);
                    oc = realign4(c1, c0, 4 - sh);
                    ov = realign4(v1, v0, 4 - sh);
                }
                __stcs(reinterpret_cast<int4 *>(out_col + qv), oc);
                __stcs(reinterpret_cast<float4 *>(out_val + qv), ov);
                continue;
            }
#pragma unroll
            for (int u = 0; u < 4; ++u) {
                const int64_t q = qv + u;
                if (q < q1) {
                    seek(q);
                    const int64_t src = ro + (q - cs);
                    cc[u] = __ldcs(chat_col + src);
                    vv[u] = __ldcs(chat_val + src);
                }
            }
            if (qv + 4 <= q1) {
                __stcs(reinterpret_cast<int4 *>(out_col + qv), make_int4(cc[0], cc[1], cc[2], cc[3]));
                __stcs(reinterpret_cast<float4 *>(out_val + qv), make_float4(vv[0], vv[1], vv[2], vv[3]));
            } else {
#pragma unroll
                for (int u = 0; u < 4; ++u)
                    if (qv + u < q1) { out_col[qv + u] = cc[u]; out_val[qv + u] = vv[u]; }
            }
        }
    }
}

}  // namespace spg
