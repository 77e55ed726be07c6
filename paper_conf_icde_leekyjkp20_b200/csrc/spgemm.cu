// C-ABI implementation (include/spgemm.h).  Host orchestration of the four stages; all
// arithmetic of the path runs in the kernels of analysis.cuh / expand.cuh / merge.cuh.
#include <cuda_runtime.h>

#include <algorithm>
#include <cmath>
#include <cstdio>
#include <cstring>
#include <string>
#include <vector>
#include <map>
#include <mutex>
#include <tuple>

#include "../../include/spgemm.h"
#include "analysis.cuh"
#include "expand.cuh"
#include "merge.cuh"
#include "merge_tiles.cuh"
#include "merge_long.cuh"
#include "scan.cuh"

using namespace spg;

// ------------------------------------------------------------------ errors ---------------
static thread_local std::string g_err;

static int fail(int code, const std::string &msg) {
    g_err = msg;
    return code;
}

#define CK(call)                                                                                 \
    do {                                                                                         \
        cudaError_t _e = (call);                                                                 \
        if (_e != cudaSuccess) {                                                                 \
            return fail(_e == cudaErrorMemoryAllocation ? SPGEMM_ERR_OUT_OF_MEMORY : SPGEMM_ERR_CUDA, \
                        std::string(#call) + ": " + cudaGetErrorString(_e));                     \
        }                                                                                        \
    } while (0)

#define TRY(...)                        \
    do {                                \
        int _r = (__VA_ARGS__);         \
        if (_r != SPGEMM_OK) return _r; \
    } while (0)

// ------------------------------------------------------------------ timing ---------------
struct TimerRec {
    const char *name;
    cudaEvent_t a, b;
};
static thread_local bool g_timing = false;
static thread_local std::vector<TimerRec> g_timers;
static thread_local std::vector<cudaEvent_t> g_event_pool;
static thread_local size_t g_events_used = 0;

static cudaEvent_t next_event() {
    if (g_events_used == g_event_pool.size()) {
        cudaEvent_t e;
        cudaEventCreate(&e);
        g_event_pool.push_back(e);
    }
    return g_event_pool[g_events_used++];
}

static void timers_reset() {
    g_timers.clear();
    g_events_used = 0;
}

struct TimedLaunch {
    cudaStream_t s;
    const char *name;
    cudaEvent_t b = nullptr;
    TimedLaunch(const char *n, cudaStream_t st) : s(st), name(n) {
        if (g_timing) {
            cudaEvent_t a = next_event();
            b = next_event();
            cudaEventRecord(a, s);
            g_timers.push_back({name, a, b});
        }
    }
    ~TimedLaunch() {
        if (g_timing) cudaEventRecord(b, s);
    }
};

#define LAUNCH(name, stream, ...)                      \
    do {                                               \
        {                                              \
            TimedLaunch _tl(name, stream);             \
            __VA_ARGS__;                               \
        }                                              \
        CK(cudaGetLastError());                        \
    } while (0)

// ------------------------------------------------------------------ memory ---------------
// One stream-ordered pool per device, created on first use under a lock (plans may be created
// from several host threads).  Its release threshold is unbounded: freed plan workspaces stay
// cached for the next plan (no driver allocation per product); spgemm_trim_pool returns them.
static cudaMemPool_t pool_for_device(int dev) {
    constexpr int kMaxDevices = 64;
    static cudaMemPool_t pools[kMaxDevices] = {};
    static std::mutex mu;
    if (dev < 0 || dev >= kMaxDevices) return nullptr;   // callers fall back to cudaMallocAsync
    std::lock_guard<std::mutex> lk(mu);
    if (!pools[dev]) {
        cudaMemPoolProps props = {};
        props.allocType = cudaMemAllocationTypePinned;
        props.handleTypes = cudaMemHandleTypeNone;
        props.location.type = cudaMemLocationTypeDevice;
        props.location.id = dev;
        cudaMemPool_t p;
        if (cudaMemPoolCreate(&p, &props) != cudaSuccess) return nullptr;
        uint64_t thr = UINT64_MAX;
        cudaMemPoolSetAttribute(p, cudaMemPoolAttrReleaseThreshold, &thr);
        pools[dev] = p;
    }
    return pools[dev];
}

struct spgemm_plan_s {
    int dev = 0;
    int num_sms = kNumSMs;
    cudaMemPool_t pool = nullptr;
    cudaStream_t last_stream = nullptr;
    spgemm_options_t opt{};
    int64_t m = 0, k = 0, n = 0, nnz_a = 0, nnz_b = 0;
    const int64_t *a_colptr = nullptr;
    const int32_t *a_rowidx = nullptr;
    const float *a_val = nullptr;
    const int64_t *b_rowptr = nullptr;
    const int32_t *b_colidx = nullptr;
    const float *b_val = nullptr;
    std::vector<void *> owned;
    int64_t bytes = 0;
    unsigned char *arena_ptr = nullptr;   // bump arena (arena_alloc)
    size_t arena_left = 0;
    // stage 1
    int64_t *work = nullptr, *rowwork = nullptr, *rowoff = nullptr, *base = nullptr;
    int32_t *deg = nullptr;
    PlanScalars *scal = nullptr;
    PlanScalars h_scal{};
    int64_t nnz_chat = 0, nnz_chat_rowwise = 0, chat_cap = 0, t_dom = 0, t_lim = 0;
    // stage 2
    int8_t *pair_cls = nullptr, *row_cls = nullptr;
    int32_t *pair_order = nullptr, *row_order = nullptr;
    int64_t pair_starts[kNumPairBuckets + 1] = {};
    int64_t row_starts[kNumRowBuckets + 1] = {};
    Piece *pieces = nullptr;       // split pieces, whole Normal blocks, gathered Low-performer blocks
    int64_t *piece_uoff = nullptr; // unit (16-byte vector) prefix over pieces
    int64_t *tile_p0 = nullptr;    // first piece of every expansion tile
    int64_t n_low = 0, n_pieces_all = 0;
    // B' (rows padded to 8 slots, row k at bp_start(b_rowptr[k], k)): cols, values
    int32_t *bp_col = nullptr;
    size_t bp_bytes = 0;
    float *bp_val = nullptr;

    int64_t n_split_pieces = 0, n_whole = 0;
    int64_t *piece_off = nullptr;
    int64_t lim_runs = 0, lim_max_deg = 0, lim_max_L = 0, nlim = 0;
    int64_t *run_start = nullptr, *run_base = nullptr;
    int32_t *run_len = nullptr, *lim_index = nullptr, *run_fill = nullptr;
    int32_t *scr_cursor = nullptr, *scr_cnt = nullptr, *scr_col = nullptr;
    float *scr_val = nullptr;
    int64_t stage_cap = 0;
    int64_t stage_cap_small = 0;   // per-block scratch of the 2 / 4 per SM limited launch
    int lim_grid = 0;
    unsigned long long *row_counter = nullptr;
    // stage 3/4
    int32_t *chat_col = nullptr;
    float *chat_val = nullptr;
    int64_t *ccount = nullptr, *crowptr = nullptr;
    int32_t *fb_rows = nullptr;
    unsigned *fb_count = nullptr;
    RowMeta *row_meta = nullptr;   // (offset, length, id) in row_order (pipelined merge bins)
    int32_t *rowmn = nullptr, *rowmx = nullptr;   // exact column range per row of C (bucket mapping)
    int64_t *row_rng = nullptr;    // (rowmn, rowmx) as int2 in row_order (pipelined bucket bins)
    bool chat_external = false;
    bool c_in_chat = false;        // C compact at the head of the Ĉ arrays (tile merge)
    int32_t *lim_defer = nullptr;     // B-Limited rows deferred to the 1-per-SM launch (limit_ctas_per_sm > 1)
    unsigned long long *unit_ticket = nullptr;   // profile buffer of the merge kernels (options.reserved[1])
    // merge tiles (merge_tiles.cuh): tile table, look-back words
    TileDesc *tiles = nullptr;
    // long rows by column groups (merge_long.cuh)
    bool long_groups = false;
    int64_t lg_groups = 0, lg_slots = 0;
    int64_t *lg_xoff = nullptr, *lg_yoff = nullptr, *lg_goff = nullptr, *lg_dense = nullptr;
    int32_t *lg_scol = nullptr, *lg_gcnt = nullptr, *lg_glo = nullptr, *lg_gnum = nullptr;
    float *lg_sval = nullptr;
    int8_t *lg_gkind = nullptr;
    unsigned long long *lg_ctr = nullptr;   // [0] row ticket, [1] dense-group count
    int64_t *tile_cnt = nullptr, *tile_base = nullptr;
    unsigned long long *tile_status = nullptr;
    int64_t tiles_max = 0;
    unsigned long long *lbi = nullptr;   // options.reserved[8] = 1: [expansion | limited merge] x kLbiSlots
    unsigned long long *exp_ticket = nullptr;   // block-path expansion claim counter
    int64_t nnz_c = -1;
    int state = 0;  // 1 planned, 2 expanded, 3 merged
};

// Plan workspaces come from a bump arena over a few large pool blocks (>= kArenaBlock bytes each,
// freed together by spgemm_destroy): ~60 workspace and temporary arrays per plan would otherwise
// cost ~130 stream-ordered malloc / free calls of host time on every product.
constexpr size_t kArenaBlock = (size_t)64 << 20;
constexpr size_t kArenaAlign = 256;

static int arena_alloc(spgemm_plan_s *p, size_t bytes, void **out, cudaStream_t s) {
    bytes = (bytes + kArenaAlign - 1) & ~(kArenaAlign - 1);
    if (p->arena_left < bytes) {
        const size_t blk = std::max(bytes, kArenaBlock);
        void *v = nullptr;
        cudaError_t e = p->pool ? cudaMallocFromPoolAsync(&v, blk, p->pool, s) : cudaMallocAsync(&v, blk, s);
        if (e != cudaSuccess)
            return fail(SPGEMM_ERR_OUT_OF_MEMORY, std::string("device allocation of ") + std::to_string(blk) +
                                                      " bytes failed: " + cudaGetErrorString(e));
        p->owned.push_back(v);
        p->bytes += (int64_t)blk;
        if (blk > bytes && blk - bytes > p->arena_left) {   // keep whichever block has more room
            p->arena_ptr = (unsigned char *)v + bytes;
            p->arena_left = blk - bytes;
        }
        *out = v;
        return SPGEMM_OK;
    }
    *out = p->arena_ptr;
    p->arena_ptr += bytes;
    p->arena_left -= bytes;
    return SPGEMM_OK;
}

template <typename T>
static int palloc(spgemm_plan_s *p, T **ptr, int64_t count, cudaStream_t s) {
    void *v = nullptr;
    TRY(arena_alloc(p, (size_t)std::max<int64_t>(count, 1) * sizeof(T), &v, s));
    *ptr = (T *)v;
    return SPGEMM_OK;
}

// temporary of a call's scope: also from the arena (released with the plan)
struct Temp {
    explicit Temp(cudaStream_t) {}
};

template <typename T>
static int talloc(spgemm_plan_s *p, Temp &, T **ptr, int64_t count) {
    return palloc(p, ptr, count, p->last_stream);
}

static inline int64_t cdiv(int64_t a, int64_t b) { return (a + b - 1) / b; }
static inline unsigned grid_for(int64_t n, int threads, int64_t cap = 148 * 64) {
    return (unsigned)std::max<int64_t>(1, std::min<int64_t>(cdiv(n, threads), cap));
}

// merge selection: default = per-bin merge + CSR compaction (merge.cuh); options.reserved[5] = 2 the
// tile merge (merge_tiles.cuh + merge_long.cuh: C placed by look-back at the head of the Ĉ arrays, no
// compaction)
static inline bool use_tile_merge(const spgemm_options_t &o) { return o.reserved[5] == 2; }
static inline bool c_in_place(const spgemm_options_t &o) { return use_tile_merge(o); }

// Large-smem kernels: opt-in shared memory size and resident blocks per SM, queried once per
// (kernel, device, smem, threads) -- these runtime calls cost host microseconds on every step.
static int kernel_occupancy(const void *kern, int smem, int threads, int *occ) {
    static std::mutex mu;
    static std::map<std::tuple<const void *, int, int, int>, int> cache;
    int dev = 0;
    CK(cudaGetDevice(&dev));
    const auto key = std::make_tuple(kern, dev, smem, threads);
    std::lock_guard<std::mutex> lk(mu);
    auto it = cache.find(key);
    if (it != cache.end()) {
        if (occ) *occ = it->second;
        return SPGEMM_OK;
    }
    CK(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
    int o = 0;
    if (threads > 0) CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&o, kern, threads, smem));
    cache[key] = o;
    if (occ) *occ = o;
    return SPGEMM_OK;
}

// ------------------------------------------------------------------ primitives -----------
template <typename Tin>
static int scan_excl(spgemm_plan_s *p, const Tin *in, int64_t n, int64_t *out, cudaStream_t s, const char *name) {
    if (n == 0) {
        CK(cudaMemsetAsync(out, 0, sizeof(int64_t), s));
        return SPGEMM_OK;
    }
    const int64_t ntiles = cdiv(n, kScanTile);
    Temp t(s);
    unsigned long long *st;   // [ntiles] look-back words + ticket
    TRY(talloc(p, t, &st, ntiles + 1));
    CK(cudaMemsetAsync(st, 0, (ntiles + 1) * 8, s));
    LAUNCH(name, s, k_scan_onepass<Tin><<<(unsigned)ntiles, kScanThreads, 0, s>>>(in, n, out, st, st + ntiles));
    return SPGEMM_OK;
}

// stable partition of [0, n) by bucket id; writes out_idx[n] and bucket starts (host) [nb+1]
static int partition(spgemm_plan_s *p, const uint8_t *bucket, int64_t n, int nb, int32_t *out_idx,
                     int64_t *d_starts, cudaStream_t s, const char *name) {
    if (n == 0) {
        CK(cudaMemsetAsync(d_starts, 0, sizeof(int64_t) * (nb + 1), s));
        return SPGEMM_OK;
    }
    const int64_t ntiles = cdiv(n, kPartThreads);
    Temp t1(s), t2(s);
    int32_t *counts;
    int64_t *offs;
    TRY(talloc(p, t1, &counts, (int64_t)nb * ntiles));
    TRY(talloc(p, t2, &offs, (int64_t)nb * ntiles + 1));
    LAUNCH(name, s, k_part_count<<<(unsigned)ntiles, kPartThreads, 0, s>>>(bucket, n, nb, counts, ntiles));
    TRY(scan_excl(p, counts, (int64_t)nb * ntiles, offs, s, name));
    LAUNCH(name, s, k_part_scatter<<<(unsigned)ntiles, kPartThreads, 0, s>>>(bucket, n, nb, offs, ntiles, out_idx));
    LAUNCH(name, s, k_bucket_starts<<<(unsigned)cdiv(nb + 1, 128), 128, 0, s>>>(offs, nb, ntiles, d_starts));
    return SPGEMM_OK;
}

#ifndef SPG_BIN_LS
#define SPG_BIN_LS 0   // (A/B build knob: 1 = twice the buckets in the 2K / 4K bins)
#endif
#ifndef SPG_WB_PIPE
#define SPG_WB_PIPE 0
#endif
#ifndef SPG_SHAPE
#define SPG_SHAPE 0   // merge-bin shapes (A/B build knob; 0 = the measured default)
#endif
// software-pipelined in-place bucket bin over rows [b0, b1) of row_order (meta table in p->row_meta)
template <int NW, int GROUPS, int EPT>
static int launch_bucket_pipe(spgemm_plan_s *p, cudaStream_t s, int64_t q0, int64_t cnt, const char *name,
                              int ctas_per_sm, bool fallback_list = true) {
    if (cnt == 0) return SPGEMM_OK;
    const int smem = BucketSmem<NW, EPT, 0>::kBytes * GROUPS;
    auto kern = k_merge_bucket_pipe<NW, GROUPS, EPT, 0>;
    int occ = 0;
    TRY(kernel_occupancy((const void *)kern, smem, NW * 32 * GROUPS, &occ));
    const int64_t grid = std::min<int64_t>(cdiv(cnt, GROUPS), (int64_t)p->num_sms * std::max(occ, 1));
    (void)ctas_per_sm;
    LAUNCH(name, s, kern<<<(unsigned)grid, NW * 32 * GROUPS, smem, s>>>(
        p->row_meta + q0, cnt, p->chat_col, p->chat_val, p->ccount, fallback_list ? p->fb_rows : nullptr, p->fb_count,
        p->row_rng ? (const int2 *)p->row_rng + q0 : nullptr));
    return SPGEMM_OK;
}

// merged rows are written in place at the head of their Ĉ bucket
template <int NW, int GROUPS, int EPT, int LS = 0>
static int launch_bucket_bin(spgemm_plan_s *p, cudaStream_t s, const int32_t *rows, int64_t cnt, const char *name,
                             int ctas_per_sm, bool fallback_list = true) {
    if (cnt == 0) return SPGEMM_OK;
    const int smem = BucketSmem<NW, EPT, LS>::kBytes * GROUPS;
    TRY(kernel_occupancy((const void *)k_merge_bucket<NW, GROUPS, EPT, LS>, smem, 0, nullptr));
    const int64_t grid = std::min<int64_t>(cdiv(cnt, GROUPS), (int64_t)p->num_sms * ctas_per_sm * 4);
    LAUNCH(name, s, k_merge_bucket<NW, GROUPS, EPT, LS><<<(unsigned)grid, NW * 32 * GROUPS, smem, s>>>(
        rows, cnt, p->rowoff, p->chat_col, p->chat_val, p->ccount, fallback_list ? p->fb_rows : nullptr, p->fb_count, 0,
        nullptr, nullptr, nullptr, p->rowmn, p->rowmx));
    return SPGEMM_OK;
}

// ------------------------------------------------------------------ ABI ------------------
// B-Limited long rows (merge.cuh k_merge_limited<NT>): limit_ctas_per_sm = 1 / 2 / 4 resident limited
// blocks per SM of 1024 / 512 / 256 threads (PAPER.md L463-L469 L, Fig. 14: the number of blocks
// an SM holds for the long rows); lim_grid = #SMs x that, persistent, rows claimed longest first.
template <int NT>
static int launch_limited_nt(spgemm_plan_s *p, cudaStream_t s, const LimitedArgs &g) {
    using C = LimCfg<NT>;
    TRY(kernel_occupancy((const void *)k_merge_limited<NT>, C::kSmem, 0, nullptr));
    LAUNCH("merge_limited_win", s, k_merge_limited<NT><<<(unsigned)p->lim_grid, NT, C::kSmem, s>>>(g));
    return SPGEMM_OK;
}

static int launch_limited(spgemm_plan_s *p, cudaStream_t s, const LimitedArgs &g0) {
    const int c = p->opt.limit_ctas_per_sm;
    if (c < 2) return launch_limited_nt<1024>(p, s, g0);
    // 2 / 4 blocks per SM; rows whose heaviest column range exceeds the smaller sorter are deferred to
    // a second, 1-per-SM launch (the heaviest rows get a whole SM's shared memory)
    LimitedArgs g = g0;
    g.stage_cap = p->stage_cap_small;
    g.coarse_cap = std::min<int64_t>(p->stage_cap_small, p->n);
    g.defer_list = p->lim_defer;
    g.defer_count = (unsigned *)(p->row_counter + 1);
    CK(cudaMemsetAsync(p->row_counter + 1, 0, 16, s));
    TRY(c >= 4 ? launch_limited_nt<256>(p, s, g) : launch_limited_nt<512>(p, s, g));
    LimitedArgs h = g0;
    h.row_counter = p->row_counter + 2;
    h.rlist = p->lim_defer;
    h.rlist_count = (const unsigned *)(p->row_counter + 1);
    const int grid = p->lim_grid;
    p->lim_grid = (int)std::min<int64_t>(p->num_sms, p->nlim);
    const int rc = launch_limited_nt<1024>(p, s, h);
    p->lim_grid = grid;
    return rc;
}

extern "C" {

int spgemm_abi_version(void) { return SPGEMM_ABI_VERSION; }

const char *spgemm_last_error(void) { return g_err.c_str(); }

void spgemm_default_options(spgemm_options_t *o) {
    if (!o) return;
    memset(o, 0, sizeof(*o));
    o->alpha = 0.0;
    o->dom_waves = 16;
    o->dom_min_work = 4096;
    o->split_ca_max = 256;
    o->piece_work = 16384;
    o->split_b_tile = 4096;
    o->beta = 0.0;
    o->limit_ctas_per_sm = 1;
    o->enable_split = 1;
    o->enable_gather = 1;
    o->enable_limit = 1;
    o->validate = 1;
}

int spgemm_trim_pool(void) {
    int dev = 0;
    CK(cudaGetDevice(&dev));
    cudaMemPool_t pool = pool_for_device(dev);
    CK(cudaDeviceSynchronize());
    if (pool) CK(cudaMemPoolTrimTo(pool, 0));
    return SPGEMM_OK;
}

int spgemm_set_timing(int32_t enable) {
    g_timing = enable != 0;
    return SPGEMM_OK;
}

int spgemm_last_timings(const char **names, float *ms, int32_t capacity, int32_t *count) {
    if (!count) return fail(SPGEMM_ERR_INVALID_ARGUMENT, "count is NULL");
    *count = (int32_t)g_timers.size();
    for (size_t q = 0; q < g_timers.size() && (int32_t)q < capacity; ++q) {
        cudaEventSynchronize(g_timers[q].b);
        float t = 0.f;
        cudaEventElapsedTime(&t, g_timers[q].a, g_timers[q].b);
        if (names) names[q] = g_timers[q].name;
        if (ms) ms[q] = t;
    }
    return SPGEMM_OK;
}

static int check_csx(int64_t nseg, int64_t other, int64_t nnz, const void *ptr, const void *idx, const void *val,
                     int32_t where, const char *what) {
    if (!ptr || (nnz > 0 && (!idx || !val)))
        return fail(SPGEMM_ERR_INVALID_ARGUMENT, std::string(what) + ": NULL array");
    if (nseg < 0 || other < 0 || nnz < 0 || nseg >= (1ll << 31) || other >= (1ll << 31))
        return fail(SPGEMM_ERR_INVALID_ARGUMENT, std::string(what) + ": bad dimensions");
    if (where != SPGEMM_DEVICE && where != SPGEMM_HOST)
        return fail(SPGEMM_ERR_INVALID_ARGUMENT, std::string(what) + ": bad `where`");
    return SPGEMM_OK;
}

static int plan_impl(spgemm_plan_s *p, const spgemm_csc_t *A, const spgemm_csr_t *B, cudaStream_t s, int64_t r0,
                     int64_t r1);

int spgemm_plan(const spgemm_csc_t *A, const spgemm_csr_t *B, const spgemm_options_t *opt, void *stream,
                spgemm_plan_t *out) {
    if (!A) return fail(SPGEMM_ERR_INVALID_ARGUMENT, "A or B is NULL");
    return spgemm_plan_rows(A, B, 0, A->nrows, opt, stream, out);
}

int spgemm_plan_rows(const spgemm_csc_t *A, const spgemm_csr_t *B, int64_t row_begin, int64_t row_end,
                     const spgemm_options_t *opt, void *stream, spgemm_plan_t *out) {
    if (!out) return fail(SPGEMM_ERR_INVALID_ARGUMENT, "plan out-pointer is NULL");
    *out = nullptr;
    if (!A || !B) return fail(SPGEMM_ERR_INVALID_ARGUMENT, "A or B is NULL");
    TRY(check_csx(A->ncols, A->nrows, A->nnz, A->colptr, A->rowidx, A->val, A->where, "A"));
    TRY(check_csx(B->nrows, B->ncols, B->nnz, B->rowptr, B->colidx, B->val, B->where, "B"));
    if (A->ncols != B->nrows) return fail(SPGEMM_ERR_INVALID_ARGUMENT, "A.ncols != B.nrows");
    if (row_begin < 0 || row_end < row_begin || row_end > A->nrows)
        return fail(SPGEMM_ERR_INVALID_ARGUMENT, "bad row window");
    int ndev = 0;
    if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev == 0) return fail(SPGEMM_ERR_NO_DEVICE, "no CUDA device");
    spgemm_plan_s *p = new spgemm_plan_s();
    if (opt) p->opt = *opt; else spgemm_default_options(&p->opt);
    spgemm_options_t d;
    spgemm_default_options(&d);
    if (p->opt.dom_waves <= 0) p->opt.dom_waves = d.dom_waves;
    if (p->opt.dom_min_work <= 0) p->opt.dom_min_work = d.dom_min_work;
    if (p->opt.split_ca_max <= 0) p->opt.split_ca_max = d.split_ca_max;
    if (p->opt.piece_work <= 0) p->opt.piece_work = d.piece_work;
    if (p->opt.split_b_tile <= 0) p->opt.split_b_tile = d.split_b_tile;
    p->opt.split_b_tile = (int32_t)pad_run(p->opt.split_b_tile);   // R4: whole 32-byte sectors (8 slots)
    if (p->opt.limit_ctas_per_sm <= 0) p->opt.limit_ctas_per_sm = d.limit_ctas_per_sm;
    int r = plan_impl(p, A, B, (cudaStream_t)stream, row_begin, row_end);
    if (r != SPGEMM_OK) {
        std::string keep = g_err;
        spgemm_destroy(p);
        g_err = keep;
        return r;
    }
    *out = p;
    return SPGEMM_OK;
}

static int upload(spgemm_plan_s *p, const void *src, int64_t bytes, int32_t where, const void **dst, cudaStream_t s) {
    if (where == SPGEMM_DEVICE) {
        *dst = src;
        return SPGEMM_OK;
    }
    unsigned char *d;
    TRY(palloc(p, &d, std::max<int64_t>(bytes, 1), s));
    if (bytes > 0) CK(cudaMemcpyAsync(d, src, (size_t)bytes, cudaMemcpyHostToDevice, s));
    *dst = d;
    return SPGEMM_OK;
}

static int plan_impl(spgemm_plan_s *p, const spgemm_csc_t *A, const spgemm_csr_t *B, cudaStream_t s, int64_t r0,
                     int64_t r1) {
    CK(cudaGetDevice(&p->dev));
    CK(cudaDeviceGetAttribute(&p->num_sms, cudaDevAttrMultiProcessorCount, p->dev));
    p->pool = pool_for_device(p->dev);
    p->last_stream = s;
    timers_reset();
    p->m = A->nrows;
    p->k = A->ncols;
    p->n = B->ncols;
    p->nnz_a = A->nnz;
    p->nnz_b = B->nnz;
    int64_t M = p->m;
    const int64_t K = p->k;
    TRY(upload(p, A->colptr, (K + 1) * 8, A->where, (const void **)&p->a_colptr, s));
    TRY(upload(p, A->rowidx, p->nnz_a * 4, A->where, (const void **)&p->a_rowidx, s));
    TRY(upload(p, A->val, p->nnz_a * 4, A->where, (const void **)&p->a_val, s));
    TRY(upload(p, B->rowptr, (K + 1) * 8, B->where, (const void **)&p->b_rowptr, s));
    TRY(upload(p, B->colidx, p->nnz_b * 4, B->where, (const void **)&p->b_colidx, s));
    TRY(upload(p, B->val, p->nnz_b * 4, B->where, (const void **)&p->b_val, s));

    TRY(palloc(p, &p->scal, 1, s));
    CK(cudaMemsetAsync(p->scal, 0, sizeof(PlanScalars), s));
    if (p->opt.validate) {
        int *flag = &p->scal->invalid;
        LAUNCH("validate", s, k_validate_ptr<<<grid_for(K + 1, 256, 1 << 30), 256, 0, s>>>(p->a_colptr, K, p->nnz_a, flag, 1));
        LAUNCH("validate", s, k_validate_ptr<<<grid_for(K + 1, 256, 1 << 30), 256, 0, s>>>(p->b_rowptr, K, p->nnz_b, flag, 2));
        PlanScalars hs;
        CK(cudaMemcpyAsync(&hs, p->scal, sizeof(hs), cudaMemcpyDeviceToHost, s));
        CK(cudaStreamSynchronize(s));
        if (hs.invalid) return fail(SPGEMM_ERR_INVALID_INPUT, "malformed colptr of A or rowptr of B");
        if (p->nnz_a > 0)
            LAUNCH("validate", s, k_validate_idx<<<grid_for(cdiv(p->nnz_a, 8), 256, 1 << 30), 256, 0, s>>>(
                p->a_colptr, p->a_rowidx, K, p->nnz_a, M, flag, 4));
        if (p->nnz_b > 0)
            LAUNCH("validate", s, k_validate_idx<<<grid_for(cdiv(p->nnz_b, 8), 256, 1 << 30), 256, 0, s>>>(
                p->b_rowptr, p->b_colidx, K, p->nnz_b, p->n, flag, 8));
        // the workload kernels below index rowwork / deg / cursors by a_rowidx: reject bad indices
        // before any of them runs (an out-of-range row would write outside the plan's arrays)
        CK(cudaMemcpyAsync(&hs, p->scal, sizeof(hs), cudaMemcpyDeviceToHost, s));
        CK(cudaStreamSynchronize(s));
        if (hs.invalid) return fail(SPGEMM_ERR_INVALID_INPUT, "malformed indices (range / order) in A or B");
    }

    // ---- row window (spgemm_plan_rows): A' = rows [r0, r1) of A, packed on the device -----
    if (r0 != 0 || r1 != A->nrows) {
        int64_t *lo, *cnt, *nptr;
        TRY(palloc(p, &lo, K, s));
        TRY(palloc(p, &cnt, K, s));
        TRY(palloc(p, &nptr, K + 1, s));
        if (K > 0)
            LAUNCH("row_window", s, k_window_count<<<grid_for(K, 256), 256, 0, s>>>(p->a_colptr, p->a_rowidx, K,
                                                                                    (int32_t)r0, (int32_t)r1, lo, cnt));
        TRY(scan_excl(p, cnt, K, nptr, s, "row_window"));
        int64_t nnz_w = 0;
        CK(cudaMemcpyAsync(&nnz_w, nptr + K, 8, cudaMemcpyDeviceToHost, s));
        CK(cudaStreamSynchronize(s));   // (the window's nnz sizes every A-entry array below)
        int32_t *widx;
        float *wval;
        TRY(palloc(p, &widx, nnz_w, s));
        TRY(palloc(p, &wval, nnz_w, s));
        if (K > 0 && nnz_w > 0)
            LAUNCH("row_window", s, k_window_copy<<<grid_for(K * 32, 256), 256, 0, s>>>(lo, nptr, K, p->a_rowidx,
                                                                                       p->a_val, (int32_t)r0, widx,
                                                                                       wval));
        p->a_colptr = nptr;
        p->a_rowidx = widx;
        p->a_val = wval;
        p->m = r1 - r0;
        p->nnz_a = nnz_w;
        M = p->m;
    }

    // ---- stage (1): workload analysis -------------------------------------------------
    TRY(palloc(p, &p->work, K, s));
    TRY(palloc(p, &p->rowwork, M, s));
    TRY(palloc(p, &p->rowoff, M + 1, s));
    TRY(palloc(p, &p->deg, M, s));
    TRY(palloc(p, &p->base, p->nnz_a, s));
    const bool col_range = p->opt.reserved[4] != 1;
    if (col_range) {
        TRY(palloc(p, &p->rowmn, M, s));
        TRY(palloc(p, &p->rowmx, M, s));
    }
    if (M > 0) {
        CK(cudaMemsetAsync(p->rowwork, 0, M * 8, s));
        CK(cudaMemsetAsync(p->deg, 0, M * 4, s));
        if (col_range) {   // empty rows keep mn > mx ("unknown")
            CK(cudaMemsetAsync(p->rowmn, 0x7f, M * 4, s));
            CK(cudaMemsetAsync(p->rowmx, 0, M * 4, s));
        }
    }
    if (K > 0)
        LAUNCH("pair_work", s, k_pair_work<<<grid_for(K, 256, p->num_sms * 8), 256, 0, s>>>(p->a_colptr, p->b_rowptr, K,
                                                                                     p->work, p->scal));
    {
        Temp tcap(s);
        int64_t *rowcap;
        TRY(talloc(p, tcap, &rowcap, M));
        if (M > 0) CK(cudaMemsetAsync(rowcap, 0, M * 8, s));
        if (p->nnz_a > 0)
            LAUNCH("row_work", s, k_row_work<<<(unsigned)cdiv(cdiv(p->nnz_a, 8), 256), 256, 0, s>>>(
                p->a_colptr, p->a_rowidx, K, p->nnz_a, p->b_rowptr, (unsigned long long *)p->rowwork, p->deg,
                (unsigned long long *)rowcap));
        TRY(scan_excl(p, rowcap, M, p->rowoff, s, "row_offsets"));   // padded bucket offsets
    }
    if (M > 0)
        LAUNCH("row_reduce", s, k_row_reduce<<<grid_for(M, 256, p->num_sms * 8), 256, 0, s>>>(p->rowwork, p->deg, M, p->scal));
    if (p->nnz_a > 0) {
        Temp tc(s);
        unsigned long long *cursor;
        TRY(talloc(p, tc, &cursor, M));
        CK(cudaMemcpyAsync(cursor, p->rowoff, M * 8, cudaMemcpyDeviceToDevice, s));
        LAUNCH("run_base", s, k_run_base<<<(unsigned)cdiv(cdiv(p->nnz_a, 8), 256), 256, 0, s>>>(
            p->a_colptr, p->a_rowidx, K, p->nnz_a, p->b_rowptr, cursor, p->base, p->rowoff, p->b_colidx, p->rowmn,
            p->rowmx));
    }
    CK(cudaMemcpyAsync(&p->h_scal, p->scal, sizeof(PlanScalars), cudaMemcpyDeviceToHost, s));
    CK(cudaMemcpyAsync(&p->chat_cap, p->rowoff + M, 8, cudaMemcpyDeviceToHost, s));
    CK(cudaStreamSynchronize(s));  // sync 1: nnz(Ĉ) both ways, Ĉ capacity, #non-empty blocks
    if (p->h_scal.invalid) return fail(SPGEMM_ERR_INVALID_INPUT, "malformed indices (range / order) in A or B");
    p->nnz_chat = (int64_t)p->h_scal.nnz_chat;
    p->nnz_chat_rowwise = (int64_t)p->h_scal.rowwise_sum;
    if (p->nnz_chat != p->nnz_chat_rowwise)
        return fail(SPGEMM_ERR_CUDA, "internal: block-wise and row-wise nnz(Ĉ) disagree");

    // thresholds (host; R1, R2, R6)
    const spgemm_options_t &o = p->opt;
    if (o.alpha > 0)
        p->t_dom = (int64_t)std::floor((double)p->nnz_chat / ((double)std::max<uint64_t>(p->h_scal.k_nonempty, 1) * o.alpha));
    else
        p->t_dom = std::min<int64_t>(o.piece_work, std::max<int64_t>(o.dom_min_work,
                                                                     cdiv(p->nnz_chat, (int64_t)p->num_sms * o.dom_waves)));
    const int64_t cap = 4096;
    if (o.beta > 0 && o.enable_limit)   // enable_limit = 0 (ablation): no Limiting rows by the paper's
        p->t_lim = std::min<int64_t>(cap, (int64_t)std::floor((double)p->nnz_chat /
                                                             ((double)std::max<uint64_t>(p->h_scal.m_nonempty, 1) * o.beta)));
    else
        p->t_lim = cap;

    // ---- stage (2): categorisation and reorganizer lists -------------------------------
    TRY(palloc(p, &p->pair_cls, K, s));
    TRY(palloc(p, &p->row_cls, M, s));
    TRY(palloc(p, &p->pair_order, K, s));
    TRY(palloc(p, &p->row_order, M, s));
    TRY(palloc(p, &p->piece_off, K + 1, s));
    int64_t *d_starts;
    TRY(palloc(p, &d_starts, kNumPairBuckets + kNumRowBuckets + 4, s));
    SplitParams sp{o.piece_work, o.split_b_tile, o.split_ca_max, o.reserved[7]};
    {
        Temp tb(s), tr(s), tn(s);
        uint8_t *pb, *rbk;
        int64_t *npieces;
        TRY(talloc(p, tb, &pb, K));
        TRY(talloc(p, tr, &rbk, M));
        TRY(talloc(p, tn, &npieces, K));
        ClassifyParams cp{p->t_dom, o.split_ca_max, o.enable_split, o.enable_gather};
        if (K > 0)
            LAUNCH("pair_classify", s, k_pair_classify<<<grid_for(K, 256), 256, 0, s>>>(p->a_colptr, p->b_rowptr, p->work, K,
                                                                                    cp, sp, p->pair_cls, pb, npieces));
        TRY(scan_excl(p, npieces, K, p->piece_off, s, "piece_scan"));
        TRY(partition(p, pb, K, kNumPairBuckets, p->pair_order, d_starts, s, "pair_partition"));
        if (M > 0)
            LAUNCH("row_classify", s, k_row_classify<<<grid_for(M, 256), 256, 0, s>>>(
                p->rowwork, p->rowoff, p->deg, M, p->t_lim, kLimitCapacity, p->row_cls, rbk, p->scal));
        TRY(partition(p, rbk, M, kNumRowBuckets, p->row_order, d_starts + kNumPairBuckets + 1, s, "row_partition"));
        CK(cudaMemcpyAsync(p->pair_starts, d_starts, sizeof(int64_t) * (kNumPairBuckets + 1), cudaMemcpyDeviceToHost, s));
        CK(cudaMemcpyAsync(p->row_starts, d_starts + kNumPairBuckets + 1, sizeof(int64_t) * (kNumRowBuckets + 1),
                           cudaMemcpyDeviceToHost, s));
        CK(cudaMemcpyAsync(&p->n_split_pieces, p->piece_off + K, 8, cudaMemcpyDeviceToHost, s));
        CK(cudaMemcpyAsync(&p->h_scal, p->scal, sizeof(PlanScalars), cudaMemcpyDeviceToHost, s));
        CK(cudaStreamSynchronize(s));  // sync 2: bin populations, #pieces, limited-row sizes
    }
    const int64_t ndom = p->pair_starts[kPairBucketSplit + 1] - p->pair_starts[kPairBucketSplit];
    p->n_whole = p->pair_starts[kPairBucketPiece + 1] - p->pair_starts[kPairBucketPiece];
    // B-Gathering blocks: the Low performers, in gather-list order (bins of 2^(n-1) < nnz(b_k*) <= 2^n)
    const int64_t g_lo = p->pair_starts[kPairBucketGather0], g_hi = p->pair_starts[kPairBucketEmpty];
    p->n_low = g_hi - g_lo;
    p->n_pieces_all = p->n_split_pieces + p->n_whole + p->n_low;
    TRY(palloc(p, &p->pieces, p->n_pieces_all, s));
    if (ndom > 0) {
        const int32_t *dom = p->pair_order + p->pair_starts[kPairBucketSplit];
        LAUNCH("piece_fill", s, k_piece_fill<<<(unsigned)cdiv(ndom * 32, 256), 256, 0, s>>>(
            dom, ndom, p->a_colptr, p->b_rowptr, sp, p->piece_off, p->pieces));
    }
    if (p->n_whole > 0)
        LAUNCH("piece_whole", s, k_piece_whole<<<grid_for(p->n_whole, 256), 256, 0, s>>>(
            p->pair_order + p->pair_starts[kPairBucketPiece], p->n_whole, p->a_colptr, p->b_rowptr,
            p->pieces + p->n_split_pieces));
    if (p->n_low > 0)
        LAUNCH("piece_whole", s, k_piece_whole<<<grid_for(p->n_low, 256), 256, 0, s>>>(
            p->pair_order + g_lo, p->n_low, p->a_colptr, p->b_rowptr, p->pieces + p->n_split_pieces + p->n_whole));
    TRY(palloc(p, &p->piece_uoff, p->n_pieces_all + 1, s));
    if (p->n_pieces_all > 0) {
        Temp tu(s);
        int64_t *units;
        TRY(talloc(p, tu, &units, p->n_pieces_all));
        LAUNCH("piece_units", s, k_piece_units<<<grid_for(p->n_pieces_all, 256), 256, 0, s>>>(
            p->pieces, p->n_pieces_all, units));
        TRY(scan_excl(p, units, p->n_pieces_all, p->piece_uoff, s, "piece_scan"));
        // (units <= nnz(Ĉ)/4 + #pieces; the tile map is sized for that bound, no host sync)
        const int64_t ntiles_max = cdiv(p->chat_cap / 4 + p->n_pieces_all, kExpTile);
        TRY(palloc(p, &p->tile_p0, ntiles_max + 1, s));
        LAUNCH("piece_scan", s, k_tile_first_piece<<<grid_for(ntiles_max + 1, 256), 256, 0, s>>>(
            p->piece_uoff, p->n_pieces_all, ntiles_max, p->tile_p0));
    } else {
        CK(cudaMemsetAsync(p->piece_uoff, 0, 8, s));
    }
    // B' = B with rows padded to 8 slots (32-byte aligned rows: vector loads, bulk copies in the expansion)
    {   // one allocation: cols then values
        const int64_t nbp = (p->nnz_b + (2 * kRunAlign - 1) * K + kRunAlign + 63) & ~(int64_t)63;   // (bp_start)
        TRY(palloc(p, &p->bp_col, 2 * nbp, s));
        p->bp_val = (float *)(p->bp_col + nbp);
        p->bp_bytes = (size_t)(2 * nbp) * 4;
    }
    if (K > 0)
        LAUNCH("pad_b", s, k_pad_b<<<grid_for(cdiv(K, 32) * 32, 256), 256, 0, s>>>(p->b_rowptr, p->b_colidx, p->b_val, K, p->bp_col,
                                                                    p->bp_val));
    // limited rows: index map, run lists, B-Limited scratch
    p->nlim = p->row_starts[kRowBucketEmpty] - p->row_starts[kRowBucketLim0];
    if (p->nlim > 0) {
        const int32_t *lrows = p->row_order + p->row_starts[kRowBucketLim0];
        TRY(palloc(p, &p->lim_index, M, s));
        TRY(palloc(p, &p->run_start, p->nlim + 1, s));
        TRY(palloc(p, &p->run_fill, p->nlim, s));
        CK(cudaMemsetAsync(p->lim_index, 0xff, M * 4, s));
        CK(cudaMemsetAsync(p->run_fill, 0, p->nlim * 4, s));
        {
            Temp tn(s);
            int64_t *nruns;
            TRY(talloc(p, tn, &nruns, p->nlim));
            LAUNCH("lim_index", s, k_lim_index<<<grid_for(p->nlim, 256), 256, 0, s>>>(lrows, p->nlim, p->deg, p->lim_index,
                                                                                  nruns));
            TRY(scan_excl(p, nruns, p->nlim, p->run_start, s, "lim_scan"));
        }
        // default merge: long rows by column groups (merge_long.cuh) when the plan has their column
        // ranges and every row fits the partition kernel's tables; else the legacy long-row kernels
        p->long_groups = use_tile_merge(o) && col_range && p->n <= (1ll << 27) &&
                         (int64_t)p->h_scal.lim_max_L <= kLongMaxL && p->opt.reserved[6] != 1;
        if (p->long_groups) {
            TRY(palloc(p, &p->lg_xoff, p->nlim + 1, s));
            TRY(palloc(p, &p->lg_yoff, p->nlim + 1, s));
            {
                Temp tx(s), ty(s);
                int64_t *xs, *ys;
                TRY(talloc(p, tx, &xs, p->nlim));
                TRY(talloc(p, ty, &ys, p->nlim));
                LAUNCH("long_sizes", s, k_long_sizes<<<grid_for(p->nlim, 256), 256, 0, s>>>(lrows, p->nlim, p->rowwork,
                                                                                           xs, ys));
                TRY(scan_excl(p, xs, p->nlim, p->lg_xoff, s, "long_sizes"));
                TRY(scan_excl(p, ys, p->nlim, p->lg_yoff, s, "long_sizes"));
            }
            // host bounds (no sync): sum pad(Lv) <= limited slots; sum of group bounds <= 4 slots / cap + 8 rows
            p->lg_slots = (int64_t)p->h_scal.lim_slots + 16;
            p->lg_groups = 4 * ((int64_t)p->h_scal.lim_slots / kGroupCap + 1) + 8 * p->nlim + 8;
            TRY(palloc(p, &p->lg_scol, p->lg_slots, s));
            TRY(palloc(p, &p->lg_sval, p->lg_slots, s));
            TRY(palloc(p, &p->lg_goff, p->lg_groups, s));
            TRY(palloc(p, &p->lg_gcnt, p->lg_groups, s));
            TRY(palloc(p, &p->lg_glo, p->lg_groups, s));
            TRY(palloc(p, &p->lg_gkind, p->lg_groups, s));
            TRY(palloc(p, &p->lg_dense, p->lg_groups, s));
            TRY(palloc(p, &p->lg_gnum, p->nlim, s));
            TRY(palloc(p, &p->lg_ctr, 2, s));
        }
        p->lim_runs = (int64_t)p->h_scal.lim_runs;
        p->lim_max_deg = (int64_t)p->h_scal.lim_max_deg;
        p->lim_max_L = (int64_t)p->h_scal.lim_max_L;
        p->lim_grid = (int)std::min<int64_t>((int64_t)p->num_sms * (o.limit_ctas_per_sm >= 4 ? 4 : o.limit_ctas_per_sm >= 2 ? 2 : 1),
                                              p->nlim);
        if (!p->long_groups) {   // legacy long-row kernels: run lists + per-CTA whole-row scratch
            TRY(palloc(p, &p->run_base, p->lim_runs, s));
            TRY(palloc(p, &p->run_len, p->lim_runs, s));
            LAUNCH("lim_runs", s, k_lim_runs<<<(unsigned)cdiv(cdiv(p->nnz_a, 8), 256), 256, 0, s>>>(
                p->a_colptr, p->a_rowidx, K, p->nnz_a, p->b_rowptr, p->base, p->lim_index, p->run_start, p->run_fill,
                p->run_base, p->run_len));
            p->stage_cap = p->lim_max_L;   // whole-row scratch (dense rows are regrouped by window)
            // 2 / 4 limited blocks per SM: their scratch is capped (rows above it are deferred to the
            // 1-per-SM launch), so the allocation stays ~#SMs x the longest row
            const int64_t nsm = std::min<int64_t>(p->num_sms, p->nlim);
            p->stage_cap_small = p->lim_grid > nsm ? std::min<int64_t>(p->lim_max_L, kLimSmallStage) : p->lim_max_L;
            const int64_t scr = std::max<int64_t>(nsm * p->stage_cap, (int64_t)p->lim_grid * p->stage_cap_small);
            TRY(palloc(p, &p->scr_cursor, (int64_t)p->lim_grid * (p->lim_max_deg + 1), s));
            TRY(palloc(p, &p->scr_cnt, (int64_t)p->lim_grid * (p->lim_max_deg + 1), s));
            p->lim_max_deg += 1;   // per-block stride of the cursor / cnt scratch (cnt holds R+1 offsets)
            TRY(palloc(p, &p->scr_col, scr, s));
            TRY(palloc(p, &p->scr_val, scr, s));
            TRY(palloc(p, &p->row_counter, 3, s));
            TRY(palloc(p, &p->lim_defer, p->nlim, s));
        }
    }
    // merge state; Ĉ itself is allocated by spgemm_expand (or is the caller's C, spgemm_execute)
    TRY(palloc(p, &p->unit_ticket, 18, s));   // [2, 18): per-phase / per-path profile (tuning)
    TRY(palloc(p, &p->ccount, M, s));
    TRY(palloc(p, &p->fb_rows, M, s));
    TRY(palloc(p, &p->fb_count, 1, s));
    TRY(palloc(p, &p->crowptr, M + 1, s));
    TRY(palloc(p, &p->exp_ticket, 1, s));
    if (p->opt.reserved[8] == 1) {   // LBI recording (Eq. (3))
        TRY(palloc(p, &p->lbi, 2 * kLbiSlots, s));
        CK(cudaMemsetAsync(p->lbi, 0, 2 * kLbiSlots * 8, s));
        CK(cudaMemsetAsync(p->lbi, 0xff, 8, s));
        CK(cudaMemsetAsync(p->lbi + kLbiSlots, 0xff, 8, s));
    }
    p->state = 1;
    return SPGEMM_OK;
}

int spgemm_expand(spgemm_plan_t p, void *stream) {
    if (!p) return fail(SPGEMM_ERR_INVALID_ARGUMENT, "plan is NULL");
    if (p->state < 1) return fail(SPGEMM_ERR_STATE, "plan not ready");
    cudaStream_t s = (cudaStream_t)stream;
    p->last_stream = s;
    CK(cudaSetDevice(p->dev));
    if (!p->chat_col) {
        TRY(palloc(p, &p->chat_col, p->chat_cap, s));
        TRY(palloc(p, &p->chat_val, p->chat_cap, s));
    }
    if (p->opt.reserved[3] == 1 && p->m > 0 && p->nnz_a > 0) {
        // row-product expansion (the paper's comparison order): A's entries by row, warp per row
        const int64_t M = p->m;
        Temp tr(s), tc(s), te(s), tk(s);
        int64_t *rptr, *list_e;
        unsigned *cursor;
        int32_t *list_k;
        TRY(talloc(p, tr, &rptr, M + 1));
        TRY(talloc(p, tc, &cursor, M));
        TRY(talloc(p, te, &list_e, p->nnz_a));
        TRY(talloc(p, tk, &list_k, p->nnz_a));
        TRY(scan_excl(p, p->deg, M, rptr, s, "expand_rows"));
        CK(cudaMemsetAsync(cursor, 0, M * 4, s));
        LAUNCH("expand_rows", s, k_row_entries<<<(unsigned)cdiv(cdiv(p->nnz_a, 8), 256), 256, 0, s>>>(
            p->a_colptr, p->k, p->nnz_a, p->a_rowidx, p->b_rowptr, rptr, cursor, list_e, list_k));
        LAUNCH("expand_rows", s, k_expand_rows<<<grid_for(M * 32, 256, (int64_t)p->num_sms * 8), 256, 0, s>>>(
            rptr, M, list_e, list_k, p->b_rowptr, p->bp_col, p->bp_val, p->a_val, p->base, p->chat_col, p->chat_val));
    } else if (p->n_pieces_all > 0) {
        // (measured: an L2 persistence window over B' -- half of L2 set aside -- made the
        // expansion 1.34 -> 2.10 ms and the compaction 1.14 -> 1.48 ms on C2; not used)
        // block path (split pieces + whole Normal blocks, TMA-staged B' tiles) unless disabled
        // (options.reserved[9] = 1: every block through the flat unit kernel, round 1's mapping)
        const int64_t nblk = p->opt.reserved[9] == 1 ? 0 : p->n_split_pieces + p->n_whole;
        if (nblk > 0) {
            CK(cudaMemsetAsync(p->exp_ticket, 0, 8, s));
            int occ = 0;
            TRY(kernel_occupancy((const void *)k_expand_blocks, kExpBlkSmem, kExpBlkThreads, &occ));
            LAUNCH("expand_blocks", s, k_expand_blocks<<<(unsigned)(p->num_sms * std::max(occ, 1)), kExpBlkThreads, kExpBlkSmem, s>>>(
                p->pieces, nblk, p->b_rowptr, p->bp_col, p->bp_val, p->a_val, p->base, p->chat_col, p->chat_val,
                p->exp_ticket, p->lbi));
        }
        // the gathered Low performers (and the rest, reserved[9] = 1): 16-byte units over fixed tiles
        // (a micro-block of W lanes per run and a run per thread measured slower: DESIGN.md §5d)
        if (nblk < p->n_pieces_all)
            LAUNCH("expand", s, k_expand_flat<<<(unsigned)p->num_sms * kExpCtasPerSM, kExpThreads, 0, s>>>(
                p->pieces, p->piece_uoff, p->n_pieces_all, p->tile_p0, p->b_rowptr, p->bp_col, p->bp_val, p->a_val,
                p->base, p->chat_col, p->chat_val, p->lbi, p->piece_uoff + nblk));
    }
    p->state = 2;
    return SPGEMM_OK;
}

static int merge_bins(spgemm_plan_s *p, cudaStream_t s) {
    const int64_t M = p->m;
    if (M > 0) {
        if (!p->row_meta) TRY(palloc(p, &p->row_meta, M, s));
        if (p->rowmn && !p->row_rng) TRY(palloc(p, &p->row_rng, M, s));
        LAUNCH("merge_meta", s, k_row_meta<<<grid_for(M, 256), 256, 0, s>>>(p->row_order, M, p->rowoff, p->rowwork,
                                                                             p->rowmn, p->rowmx, p->row_meta,
                                                                             (int2 *)p->row_rng));
    }
    if (M > 0) CK(cudaMemsetAsync(p->ccount, 0, M * 8, s));
    auto rows_of = [&](int b0, int b1, int64_t *cnt) {
        *cnt = p->row_starts[b1] - p->row_starts[b0];
        return p->row_order + p->row_starts[b0];
    };
    int64_t cnt;
    const int32_t *rows = rows_of(kRowBucketPass, kRowBucketPass + 1, &cnt);
    if (cnt > 0)
        LAUNCH("merge_pass", s, k_merge_pass<<<grid_for(cnt, 256), 256, 0, s>>>(rows, cnt, p->rowwork, p->ccount));
    rows = rows_of(kRowBucketWarp, kRowBucketWarp + 1, &cnt);
    if (cnt > 0)
        LAUNCH("merge_warp", s, k_merge_warp<<<(unsigned)cdiv(cnt * 32, 256), 256, 0, s>>>(
            rows, cnt, p->rowoff, p->chat_col, p->chat_val, p->ccount, nullptr, nullptr, nullptr));
    CK(cudaMemsetAsync(p->fb_count, 0, sizeof(unsigned), s));
    // <= 256 slots: a warp per row, bucket sort (C4 merge 2.02 -> 1.68 ms, C5 2.80 -> 2.49 ms vs the
    // software-pipelined warp merge path, kept as reserved[11] = 1); <= 1024: pipelined per-row bucket sort;
    // <= 4096: per-row bucket sort (8 / 16 warps).  (The slower alternatives measured in round 1 --
    // register-staged counting sort, bucket sort or merge path everywhere, register bitonic, the
    // bucket-owner walk, the fused unit merge -- were removed in round 2.)
    rows = rows_of(kRowBucketWarp64, kRowBucketSort256 + 1, &cnt);   // 32 < slots <= 256
    if (p->opt.reserved[11] != 1) {   // warp-per-row bucket sort, 64 / 128 / 256-slot sorters (default;
                                      // reserved[11] = 1: the warp merge path, round 1)
        int64_t c1;
        const int32_t *r1 = rows_of(kRowBucketWarp64, kRowBucketWarp64 + 1, &c1);
#if SPG_WB_PIPE   // (A/B build knob: software-pipelined warp-per-row bins)
        TRY(launch_bucket_pipe<1, 8, 2>(p, s, p->row_starts[kRowBucketWarp64], c1, "merge_wbucket64", 8));
        r1 = rows_of(kRowBucketWarp128, kRowBucketWarp128 + 1, &c1);
        TRY(launch_bucket_pipe<1, 8, 4>(p, s, p->row_starts[kRowBucketWarp128], c1, "merge_wbucket128", 8));
        r1 = rows_of(kRowBucketSort256, kRowBucketSort256 + 1, &c1);
        TRY(launch_bucket_pipe<1, 8, 8>(p, s, p->row_starts[kRowBucketSort256], c1, "merge_wbucket256", 8));
#else
        TRY(launch_bucket_bin<1, 8, 2>(p, s, r1, c1, "merge_wbucket64", 8));
        r1 = rows_of(kRowBucketWarp128, kRowBucketWarp128 + 1, &c1);
        TRY(launch_bucket_bin<1, 8, 4>(p, s, r1, c1, "merge_wbucket128", 8));
        r1 = rows_of(kRowBucketSort256, kRowBucketSort256 + 1, &c1);
        TRY(launch_bucket_bin<1, 8, 8>(p, s, r1, c1, "merge_wbucket256", 8));
#endif
        cnt = 0;
    }
    if (cnt > 0) {
        constexpr int G = 8;
        const int smem = WmpSmem<256>::kBytes * G;
        int occ = 0;
        TRY(kernel_occupancy((const void *)k_merge_wmp_pipe<G>, smem, 32 * G, &occ));
        const int64_t q0 = p->row_starts[kRowBucketWarp64];
        const int64_t grid = std::min<int64_t>(cdiv(cnt, G), (int64_t)p->num_sms * std::max(occ, 1));
        LAUNCH("merge_wmp256", s, k_merge_wmp_pipe<G><<<(unsigned)grid, 32 * G, smem, s>>>(
            p->row_meta + q0, cnt, p->chat_col, p->chat_val, p->ccount));
    }
    {
        const int64_t q = p->row_starts[kRowBucketSort512];
#if SPG_SHAPE == 1   // (A/B build knob: more threads per row, fewer slots per thread)
        TRY(launch_bucket_pipe<4, 2, 4>(p, s, q, p->row_starts[kRowBucketSort512 + 1] - q, "merge_bucket512", 8));
#else
        TRY(launch_bucket_pipe<2, 4, 8>(p, s, q, p->row_starts[kRowBucketSort512 + 1] - q, "merge_bucket512", 8));
#endif
        const int64_t q2 = p->row_starts[kRowBucketSort1K];
#if SPG_SHAPE == 1
        TRY(launch_bucket_pipe<8, 1, 4>(p, s, q2, p->row_starts[kRowBucketSort1K + 1] - q2, "merge_bucket1k", 8));
#else
        TRY(launch_bucket_pipe<4, 2, 8>(p, s, q2, p->row_starts[kRowBucketSort1K + 1] - q2, "merge_bucket1k", 8));
#endif
    }
    rows = rows_of(kRowBucketSort2K, kRowBucketSort2K + 1, &cnt);
#if SPG_SHAPE == 2   // (A/B build knob: software-pipelined 2K / 4K bins)
    {
        const int64_t qa = p->row_starts[kRowBucketSort2K];
        TRY(launch_bucket_pipe<8, 1, 8>(p, s, qa, cnt, "merge_bucket2k", 4));
    }
#else
    TRY(launch_bucket_bin<8, 1, 8, SPG_BIN_LS>(p, s, rows, cnt, "merge_bucket2k", 8));
#endif
    rows = rows_of(kRowBucketSort4K, kRowBucketSort4K + 1, &cnt);
#if SPG_SHAPE == 2
    {
        const int64_t qb = p->row_starts[kRowBucketSort4K];
        TRY(launch_bucket_pipe<16, 1, 8>(p, s, qb, cnt, "merge_bucket4k", 2));
    }
#else
    TRY(launch_bucket_bin<16, 1, 8, SPG_BIN_LS>(p, s, rows, cnt, "merge_bucket4k", 4));
#endif
    {   // rows whose buckets overflowed: natural merge sort (count read on the device)
        constexpr int CAP = 4096;
        const int smem = SortSmem<CAP>::kBytes;
        TRY(kernel_occupancy((const void *)k_merge_rows<8, 1, CAP>, smem, 0, nullptr));
        LAUNCH("merge_fallback", s, k_merge_rows<8, 1, CAP><<<(unsigned)p->num_sms * 2, 256, smem, s>>>(
            p->fb_rows, 0, p->rowoff, p->rowwork, p->chat_col, p->chat_val, p->ccount, p->fb_count, nullptr, nullptr,
            nullptr));
    }
    if (p->nlim > 0) {
        CK(cudaMemsetAsync(p->row_counter, 0, 8, s));
        LimitedArgs g{};
        g.rows = p->row_order + p->row_starts[kRowBucketLim0];
        g.nrows = p->nlim;
        g.rowoff = p->rowoff;
        g.rowwork = p->rowwork;
        g.run_start = p->run_start;
        g.run_base = p->run_base;
        g.run_len = p->run_len;
        g.chat_col = p->chat_col;
        g.chat_val = p->chat_val;
        g.ccount = p->ccount;
        g.scratch_cursor = p->scr_cursor;
        g.scratch_cnt = p->scr_cnt;
        g.scratch_col = p->scr_col;
        g.scratch_val = p->scr_val;
        g.max_deg = p->lim_max_deg;
        g.stage_cap = p->stage_cap;
        g.row_counter = p->row_counter;
        g.out_col = nullptr;   // merged in place
        g.out_val = nullptr;
        g.out_off = nullptr;
        g.skip_small = 1;
        g.prof = p->opt.reserved[1] == 3 ? p->unit_ticket + 2 : nullptr;
        if (g.prof) CK(cudaMemsetAsync(g.prof, 0, 16 * 8, s));
        g.coarse_cap = std::min<int64_t>(p->stage_cap, p->n);
        g.lbi = p->lbi ? p->lbi + kLbiSlots : nullptr;
        g.dense_div = p->opt.reserved[12] > 0 ? p->opt.reserved[12] : 4;   // (tuning knob)
        // limited rows whose bucket fits 9216 slots: one 1024-thread bucket-sort CTA per SM
        // (B-Limiting: 213 KB of shared memory each); the others: windowed kernel below
        // limited rows of <= 9216 slots: software-pipelined 1024-thread bucket sort, the next row's slots
        // loaded while this one sorts (C5 20.9 -> 20.0 ms, C3 14.9 -> 14.0 ms vs the plain bin)
        TRY(launch_bucket_pipe<32, 1, 9>(p, s, p->row_starts[kRowBucketLim0], g.nrows, "merge_limited_smem", 1, false));
        TRY(launch_limited(p, s, g));
    }
    TRY(scan_excl(p, p->ccount, M, p->crowptr, s, "c_rowptr"));
    return SPGEMM_OK;
}

// B-Limited rows (merge.cuh): merged in place at the head of their Ĉ bucket, ccount[i] = length
static int merge_limited_in_place(spgemm_plan_s *p, cudaStream_t s) {
    if (p->nlim == 0) return SPGEMM_OK;
    CK(cudaMemsetAsync(p->row_counter, 0, 8, s));
    LimitedArgs g{};
    g.rows = p->row_order + p->row_starts[kRowBucketLim0];
    g.nrows = p->nlim;
    g.rowoff = p->rowoff;
    g.rowwork = p->rowwork;
    g.run_start = p->run_start;
    g.run_base = p->run_base;
    g.run_len = p->run_len;
    g.chat_col = p->chat_col;
    g.chat_val = p->chat_val;
    g.ccount = p->ccount;
    g.scratch_cursor = p->scr_cursor;
    g.scratch_cnt = p->scr_cnt;
    g.scratch_col = p->scr_col;
    g.scratch_val = p->scr_val;
    g.max_deg = p->lim_max_deg;
    g.stage_cap = p->stage_cap;
    g.row_counter = p->row_counter;
    g.out_col = nullptr;   // merged in place
    g.out_val = nullptr;
    g.out_off = nullptr;
    g.skip_small = 1;
    g.prof = p->opt.reserved[1] == 3 ? p->unit_ticket + 2 : nullptr;
    if (g.prof) CK(cudaMemsetAsync(g.prof, 0, 16 * 8, s));
    g.coarse_cap = std::min<int64_t>(p->stage_cap, p->n);
    g.lbi = p->lbi ? p->lbi + kLbiSlots : nullptr;
        g.dense_div = p->opt.reserved[12] > 0 ? p->opt.reserved[12] : 4;   // (tuning knob)
    // limited rows whose bucket fits 9216 slots: one 1024-thread bucket-sort CTA per SM
    // (B-Limiting: 213 KB of shared memory each); the others: windowed kernel below
    TRY(launch_bucket_bin<32, 1, 9>(p, s, g.rows, g.nrows, "merge_limited_smem", 1, false));
    TRY(launch_limited(p, s, g));
    return SPGEMM_OK;
}

// Default merge (merge_tiles.cuh): B-Limited rows in place, then one persistent kernel over the tiles
// (short-row groups and long-row chunks) in row order, C placed by look-back at the head of Ĉ.
static int merge_tiles_path(spgemm_plan_s *p, cudaStream_t s) {
    const int64_t M = p->m;
    if (M == 0) {
        CK(cudaMemsetAsync(p->crowptr, 0, 8, s));
        return SPGEMM_OK;
    }
    CK(cudaMemsetAsync(p->ccount, 0, M * 8, s));
    LongTables lt{};
    if (p->nlim > 0 && p->long_groups) {
        // B-Limited rows: column-group partition (limit_ctas_per_sm partition CTAs per SM, longest
        // rows first), then the dense groups merged in place in the scratch
        CK(cudaMemsetAsync(p->lg_ctr, 0, 16, s));
        LongArgs la;
        la.rows = p->row_order + p->row_starts[kRowBucketLim0];
        la.nrows = p->nlim;
        la.rowoff = p->rowoff;
        la.rowwork = p->rowwork;
        la.rowmn = p->rowmn;
        la.rowmx = p->rowmx;
        la.col = p->chat_col;
        la.val = p->chat_val;
        la.xoff = p->lg_xoff;
        la.yoff = p->lg_yoff;
        la.scol = p->lg_scol;
        la.sval = p->lg_sval;
        la.g_off = p->lg_goff;
        la.g_cnt = p->lg_gcnt;
        la.g_lo = p->lg_glo;
        la.g_kind = p->lg_gkind;
        la.g_num = p->lg_gnum;
        la.dense_list = p->lg_dense;
        la.dense_count = p->lg_ctr + 1;
        la.counter = p->lg_ctr;
        int occ = 0;
        TRY(kernel_occupancy((const void *)k_long_partition, kPartSmem, kPartT, &occ));
        const int64_t grid = std::min<int64_t>((int64_t)p->num_sms * std::min(std::max(occ, 1), p->opt.limit_ctas_per_sm),
                                               p->nlim);
        LAUNCH("merge_long_partition", s, k_long_partition<<<(unsigned)grid, kPartT, kPartSmem, s>>>(la));
        TRY(kernel_occupancy((const void *)k_long_dense, kDenseSmem, kDenseT, nullptr));
        LAUNCH("merge_long_dense", s, k_long_dense<<<(unsigned)p->num_sms, kDenseT, kDenseSmem, s>>>(
            p->lg_dense, p->lg_ctr + 1, p->lg_goff, p->lg_gcnt, p->lg_glo, p->lg_gkind, p->lg_scol, p->lg_sval));
        lt.lim_index = p->lim_index;
        lt.yoff = p->lg_yoff;
        lt.g_num = p->lg_gnum;
        lt.g_off = p->lg_goff;
        lt.g_cnt = p->lg_gcnt;
        lt.g_kind = p->lg_gkind;
    } else {
        TRY(merge_limited_in_place(p, s));
    }
    const int64_t nch = cdiv(M, kTileRowChunk);
    if (!p->tiles) {
        // short tiles <= M; long-row tiles <= groups + merged chunks (<= groups + slots / chunk), or
        // in-place chunks <= nlim + nnz(Ĉ) / kCopyChunk
        p->tiles_max = M + p->nlim + p->chat_cap / kCopyChunk + 2 * p->lg_groups + 1;
        TRY(palloc(p, &p->tiles, p->tiles_max, s));
        TRY(palloc(p, &p->tile_cnt, nch, s));
        TRY(palloc(p, &p->tile_base, nch + 1, s));
        TRY(palloc(p, &p->tile_status, p->tiles_max + 2, s));
    }
    LAUNCH("merge_tiles_table", s, k_tile_table<false><<<(unsigned)cdiv(nch * 32, 128), 128, 0, s>>>(
        p->rowoff, p->row_cls, p->ccount, lt, M, p->tile_cnt, nullptr, nullptr));
    TRY(scan_excl(p, p->tile_cnt, nch, p->tile_base, s, "merge_tiles_table"));
    LAUNCH("merge_tiles_table", s, k_tile_table<true><<<(unsigned)cdiv(nch * 32, 128), 128, 0, s>>>(
        p->rowoff, p->row_cls, p->ccount, lt, M, nullptr, p->tile_base, p->tiles));
    CK(cudaMemsetAsync(p->tile_status, 0, (p->tiles_max + 2) * 8, s));
    TileArgs ta;
    ta.tiles = p->tiles;
    ta.ntiles = p->tile_base + nch;
    ta.rowoff = p->rowoff;
    ta.rowwork = p->rowwork;
    ta.ccount = p->ccount;
    ta.col = p->chat_col;
    ta.val = p->chat_val;
    ta.crowptr = p->crowptr;
    ta.M = M;
    ta.status = p->tile_status;
    ta.ticket = p->tile_status + p->tiles_max + 1;
    ta.lt = lt;
    ta.scol = p->lg_scol;
    ta.sval = p->lg_sval;
    ta.debug = p->opt.reserved[1];
    ta.prof = p->unit_ticket + 2;
    if (ta.debug == 2) CK(cudaMemsetAsync(ta.prof, 0, 16 * 8, s));
    using TS = TileSmem<kTileThreads, kTileEPT>;
    auto kern = k_merge_tiles<kTileThreads, kTileEPT>;
    int occ = 0;
    TRY(kernel_occupancy((const void *)kern, TS::kBytes, kTileThreads, &occ));
    LAUNCH("merge_tiles", s, kern<<<(unsigned)(p->num_sms * std::max(occ, 1)), kTileThreads, TS::kBytes, s>>>(ta));
    return SPGEMM_OK;
}

int spgemm_merge(spgemm_plan_t p, void *stream, int64_t *nnz_c) {
    if (!p) return fail(SPGEMM_ERR_INVALID_ARGUMENT, "plan is NULL");
    if (p->state < 2) return fail(SPGEMM_ERR_STATE, "spgemm_merge before spgemm_expand");
    if (p->state >= 3) return fail(SPGEMM_ERR_STATE, "plan already merged (plans are single-use)");
    cudaStream_t s = (cudaStream_t)stream;
    p->last_stream = s;
    CK(cudaSetDevice(p->dev));
    const int64_t M = p->m;
    p->c_in_chat = c_in_place(p->opt);
    if (use_tile_merge(p->opt)) TRY(merge_tiles_path(p, s));
    else TRY(merge_bins(p, s));
    CK(cudaMemcpyAsync(&p->nnz_c, p->crowptr + M, 8, cudaMemcpyDeviceToHost, s));
    CK(cudaStreamSynchronize(s));
    p->state = 3;
    if (nnz_c) *nnz_c = p->nnz_c;
    return SPGEMM_OK;
}

int spgemm_output(spgemm_plan_t p, spgemm_csr_out_t *C, void *stream) {
    if (!p || !C) return fail(SPGEMM_ERR_INVALID_ARGUMENT, "plan or C is NULL");
    if (p->state < 3) return fail(SPGEMM_ERR_STATE, "spgemm_output before spgemm_merge");
    if (!C->rowptr || (p->nnz_c > 0 && (!C->colidx || !C->val)))
        return fail(SPGEMM_ERR_INVALID_ARGUMENT, "C arrays are NULL");
    cudaStream_t s = (cudaStream_t)stream;
    p->last_stream = s;
    CK(cudaSetDevice(p->dev));
    C->nrows = p->m;
    C->ncols = p->n;
    C->nnz = p->nnz_c;
    const int64_t nnz = p->nnz_c;
    if (p->c_in_chat) {
        // tile merge: C is compact at the head of the Ĉ arrays (merge_tiles.cuh)
        const cudaMemcpyKind kind = C->where == SPGEMM_HOST ? cudaMemcpyDeviceToHost : cudaMemcpyDeviceToDevice;
        CK(cudaMemcpyAsync(C->rowptr, p->crowptr, (p->m + 1) * 8, kind, s));
        if (nnz > 0 && C->colidx != p->chat_col) {
            CK(cudaMemcpyAsync(C->colidx, p->chat_col, nnz * 4, kind, s));
            CK(cudaMemcpyAsync(C->val, p->chat_val, nnz * 4, kind, s));
        }
        if (C->where == SPGEMM_HOST) CK(cudaStreamSynchronize(s));
        return SPGEMM_OK;
    }
    // per-bin merge: rows merged in place in their Ĉ buckets -> CSR compaction
    int32_t *dcol = C->colidx;
    float *dval = C->val;
    Temp t1(s), t2(s);
    if (C->where == SPGEMM_HOST) {
        TRY(talloc(p, t1, &dcol, nnz));
        TRY(talloc(p, t2, &dval, nnz));
    }
    const bool aligned = ((uintptr_t)dcol & 15) == 0 && ((uintptr_t)dval & 15) == 0;
    if (nnz > 0 && aligned && p->opt.reserved[2] != 1) {
        // load-balanced by output entry (any row-length mix)
        const int64_t nchunks = cdiv(nnz, kCmpChunk);
        Temp tc(s);
        int32_t *chunk_r0;
        TRY(talloc(p, tc, &chunk_r0, nchunks + 1));
        LAUNCH("compact", s, k_chunk_first_row<<<grid_for(nchunks + 1, 256), 256, 0, s>>>(p->crowptr, p->m, nnz, nchunks,
                                                                                          chunk_r0));
        LAUNCH("compact", s, k_compact_flat<<<(unsigned)std::min<int64_t>(nchunks, (int64_t)p->num_sms * 8), kCmpThreads, 0,
                                              s>>>(p->crowptr, p->rowoff, chunk_r0, nnz, nchunks, p->chat_col,
                                                   p->chat_val, dcol, dval));
    } else if (nnz > 0) {
        // warp per row (realigned vectors) + CTA per long row (unaligned caller buffers; tuning)
        LAUNCH("compact", s, k_compact_rows<<<grid_for(p->m * 32, 256, (int64_t)p->num_sms * 16), 256, 0, s>>>(
            nullptr, p->crowptr, p->m, p->rowoff, p->chat_col, p->chat_val, dcol, dval));
        if (p->nlim > 0)
            LAUNCH("compact", s, k_compact_long<<<(unsigned)std::min<int64_t>(p->nlim, (int64_t)p->num_sms * 4),
                                                   kCompactLongThreads, 0, s>>>(
                p->row_order + p->row_starts[kRowBucketLim0], p->nlim, p->crowptr, p->rowoff, p->chat_col,
                p->chat_val, dcol, dval));
    }
    if (C->where == SPGEMM_HOST) {
        CK(cudaMemcpyAsync(C->rowptr, p->crowptr, (p->m + 1) * 8, cudaMemcpyDeviceToHost, s));
        if (nnz > 0) {
            CK(cudaMemcpyAsync(C->colidx, dcol, nnz * 4, cudaMemcpyDeviceToHost, s));
            CK(cudaMemcpyAsync(C->val, dval, nnz * 4, cudaMemcpyDeviceToHost, s));
        }
        CK(cudaStreamSynchronize(s));
    } else {
        CK(cudaMemcpyAsync(C->rowptr, p->crowptr, (p->m + 1) * 8, cudaMemcpyDeviceToDevice, s));
    }
    return SPGEMM_OK;
}

int spgemm_execute(spgemm_plan_t p, spgemm_alloc_fn alloc, void *ctx, int32_t out_where, spgemm_csr_out_t *C,
                   void *stream) {
    if (!p || !alloc || !C) return fail(SPGEMM_ERR_INVALID_ARGUMENT, "plan, alloc or C is NULL");
    if (out_where != SPGEMM_DEVICE && out_where != SPGEMM_HOST)
        return fail(SPGEMM_ERR_INVALID_ARGUMENT, "bad out_where");
    if (p->state != 1) return fail(SPGEMM_ERR_STATE, "spgemm_execute needs a fresh plan");
    C->where = out_where;
    if (out_where == SPGEMM_DEVICE && c_in_place(p->opt)) {
        // device C: its column / value arrays (capacity nnz(Ĉ) slots) hold Ĉ during the merge and
        // C at their head afterwards -- no copy, no second nnz(Ĉ)-sized buffer
        C->rowptr = (int64_t *)alloc((size_t)(p->m + 1) * 8, out_where, ctx);
        C->colidx = (int32_t *)alloc((size_t)std::max<int64_t>(p->chat_cap, 1) * 4, out_where, ctx);
        C->val = (float *)alloc((size_t)std::max<int64_t>(p->chat_cap, 1) * 4, out_where, ctx);
        if (!C->rowptr || !C->colidx || !C->val) return fail(SPGEMM_ERR_OUT_OF_MEMORY, "C allocation callback failed");
        p->chat_col = C->colidx;
        p->chat_val = C->val;
        p->chat_external = true;
        TRY(spgemm_expand(p, stream));
        int64_t nnz;
        TRY(spgemm_merge(p, stream, &nnz));
        return spgemm_output(p, C, stream);
    }
    TRY(spgemm_expand(p, stream));
    int64_t nnz;
    TRY(spgemm_merge(p, stream, &nnz));
    C->rowptr = (int64_t *)alloc((size_t)(p->m + 1) * 8, out_where, ctx);
    C->colidx = (int32_t *)alloc((size_t)std::max<int64_t>(nnz, 1) * 4, out_where, ctx);
    C->val = (float *)alloc((size_t)std::max<int64_t>(nnz, 1) * 4, out_where, ctx);
    if (!C->rowptr || !C->colidx || !C->val) return fail(SPGEMM_ERR_OUT_OF_MEMORY, "C allocation callback failed");
    return spgemm_output(p, C, stream);
}

int spgemm_get_stats(spgemm_plan_t p, spgemm_stats_t *st) {
    if (!p || !st) return fail(SPGEMM_ERR_INVALID_ARGUMENT, "plan or stats is NULL");
    memset(st, 0, sizeof(*st));
    st->m = p->m;
    st->k = p->k;
    st->n = p->n;
    st->nnz_a = p->nnz_a;
    st->nnz_b = p->nnz_b;
    st->nnz_chat = p->nnz_chat;
    st->nnz_chat_rowwise = p->nnz_chat_rowwise;
    st->nnz_c = p->nnz_c;
    st->k_nonempty = (int64_t)p->h_scal.k_nonempty;
    st->m_nonempty = (int64_t)p->h_scal.m_nonempty;
    st->t_dom = p->t_dom;
    st->t_lim = p->t_lim;
    st->n_dominator = p->pair_starts[kPairBucketSplit + 1] - p->pair_starts[kPairBucketSplit];
    st->n_normal = p->n_whole;
    st->n_low = p->pair_starts[kPairBucketEmpty] - p->pair_starts[kPairBucketGather0];
    st->n_pieces_split = p->n_split_pieces;
    for (int b = 0; b < 6; ++b)
        st->n_gather_bin[b] = p->pair_starts[kPairBucketGather0 + b * 16 + 16] - p->pair_starts[kPairBucketGather0 + b * 16];
    st->n_rows_bin[0] = p->row_starts[kRowBucketEmpty + 1] - p->row_starts[kRowBucketEmpty];
    st->n_rows_bin[1] = p->row_starts[kRowBucketPass + 1] - p->row_starts[kRowBucketPass];
    st->n_rows_bin[2] = p->row_starts[kRowBucketWarp + 1] - p->row_starts[kRowBucketWarp];
    st->n_rows_bin[3] = p->row_starts[kRowBucketSort1K + 1] - p->row_starts[kRowBucketWarp64];
    st->n_rows_bin[4] = p->row_starts[kRowBucketSort4K + 1] - p->row_starts[kRowBucketSort2K];
    st->n_rows_bin[5] = p->nlim;
    st->bytes_workspace = p->bytes;
    st->n_units = st->n_units_fallback = -1;
    if (p->state >= 3 && p->m > 0 && p->tiles) {   // tile merge: number of tiles walked
        CK(cudaMemcpy(&st->n_units, p->tile_base + cdiv(p->m, kTileRowChunk), 8, cudaMemcpyDeviceToHost));
        st->n_units_fallback = 0;
    }
    return SPGEMM_OK;
}

int spgemm_inspect(spgemm_plan_t p, int32_t what, void *dst, int64_t cap, int64_t *size) {
    if (!p || !size) return fail(SPGEMM_ERR_INVALID_ARGUMENT, "plan or size is NULL");
    CK(cudaSetDevice(p->dev));
    CK(cudaDeviceSynchronize());
    const void *src = nullptr;
    int64_t bytes = 0;
    std::vector<int64_t> tmp;
    switch (what) {
        case SPGEMM_VIEW_WORK: src = p->work; bytes = p->k * 8; break;
        case SPGEMM_VIEW_ROWWORK: src = p->rowwork; bytes = p->m * 8; break;
        case SPGEMM_VIEW_ROWOFF: src = p->rowoff; bytes = (p->m + 1) * 8; break;
        case SPGEMM_VIEW_PAIR_CLASS: src = p->pair_cls; bytes = p->k; break;
        case SPGEMM_VIEW_ROW_CLASS: src = p->row_cls; bytes = p->m; break;
        case SPGEMM_VIEW_ROW_COLMIN: src = p->rowmn; bytes = p->rowmn ? p->m * 4 : 0; break;
        case SPGEMM_VIEW_ROW_COLMAX: src = p->rowmx; bytes = p->rowmx ? p->m * 4 : 0; break;
        case SPGEMM_VIEW_CHAT_COL:
            if (p->state != 2) return fail(SPGEMM_ERR_STATE, "Ĉ is only inspectable between expand and merge");
            src = p->chat_col; bytes = p->chat_cap * 4; break;
        case SPGEMM_VIEW_CHAT_VAL:
            if (p->state != 2) return fail(SPGEMM_ERR_STATE, "Ĉ is only inspectable between expand and merge");
            src = p->chat_val; bytes = p->chat_cap * 4; break;
        case SPGEMM_VIEW_CROWPTR:
            if (p->state < 3) return fail(SPGEMM_ERR_STATE, "C row pointers exist after merge");
            src = p->crowptr; bytes = (p->m + 1) * 8; break;
        case SPGEMM_VIEW_LBI:
            src = p->lbi; bytes = p->lbi ? 2 * kLbiSlots * 8 : 0; break;
        case SPGEMM_VIEW_UNIT_PROFILE:
            if (p->state < 3) return fail(SPGEMM_ERR_STATE, "the unit profile exists after merge");
            src = p->unit_ticket + 2; bytes = 16 * 8; break;
        case SPGEMM_VIEW_GATHER: {
            const int64_t lo = p->pair_starts[kPairBucketGather0], hi = p->pair_starts[kPairBucketEmpty];
            src = p->pair_order + lo;
            bytes = (hi - lo) * 4;
            break;
        }
        case SPGEMM_VIEW_PIECES: {
            bytes = p->n_split_pieces * 5 * 8;
            *size = bytes;
            if (cap < bytes) return fail(SPGEMM_ERR_INVALID_ARGUMENT, "capacity too small");
            std::vector<Piece> hp((size_t)p->n_split_pieces);
            if (p->n_split_pieces) CK(cudaMemcpy(hp.data(), p->pieces, hp.size() * sizeof(Piece), cudaMemcpyDeviceToHost));
            int64_t *o = (int64_t *)dst;
            for (size_t q = 0; q < hp.size(); ++q) {
                o[q * 5 + 0] = hp[q].k;
                o[q * 5 + 1] = hp[q].a_lo;
                o[q * 5 + 2] = hp[q].a_lo + hp[q].a_len;
                o[q * 5 + 3] = hp[q].b_lo;
                o[q * 5 + 4] = hp[q].b_lo + hp[q].b_len;
            }
            return SPGEMM_OK;
        }
        default: return fail(SPGEMM_ERR_INVALID_ARGUMENT, "unknown view");
    }
    *size = bytes;
    if (cap < bytes) return fail(SPGEMM_ERR_INVALID_ARGUMENT, "capacity too small");
    if (bytes > 0) CK(cudaMemcpy(dst, src, (size_t)bytes, cudaMemcpyDeviceToHost));
    return SPGEMM_OK;
}

int spgemm_row_partition(const spgemm_csc_t *A, const spgemm_csr_t *B, int32_t parts, int64_t *bounds_host,
                         void *stream) {
    if (!A || !B || !bounds_host || parts < 1) return fail(SPGEMM_ERR_INVALID_ARGUMENT, "bad row_partition arguments");
    TRY(check_csx(A->ncols, A->nrows, A->nnz, A->colptr, A->rowidx, A->val, A->where, "A"));
    TRY(check_csx(B->nrows, B->ncols, B->nnz, B->rowptr, B->colidx, B->val, B->where, "B"));
    if (A->ncols != B->nrows) return fail(SPGEMM_ERR_INVALID_ARGUMENT, "A.ncols != B.nrows");
    int ndev = 0;
    if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev == 0) return fail(SPGEMM_ERR_NO_DEVICE, "no CUDA device");
    spgemm_plan_s tmp;
    spgemm_plan_s *p = &tmp;
    cudaStream_t s = (cudaStream_t)stream;
    CK(cudaGetDevice(&p->dev));
    p->pool = pool_for_device(p->dev);
    p->last_stream = s;
    const int64_t M = A->nrows, K = A->ncols;
    int r = [&]() -> int {
        TRY(upload(p, A->colptr, (K + 1) * 8, A->where, (const void **)&p->a_colptr, s));
        TRY(upload(p, A->rowidx, A->nnz * 4, A->where, (const void **)&p->a_rowidx, s));
        TRY(upload(p, B->rowptr, (K + 1) * 8, B->where, (const void **)&p->b_rowptr, s));
        TRY(palloc(p, &p->rowwork, M, s));
        TRY(palloc(p, &p->deg, M, s));
        TRY(palloc(p, &p->rowoff, M + 1, s));
        int64_t *bounds;
        TRY(palloc(p, &bounds, parts + 1, s));
        if (M > 0) {
            CK(cudaMemsetAsync(p->rowwork, 0, M * 8, s));
            CK(cudaMemsetAsync(p->deg, 0, M * 4, s));
        }
        if (A->nnz > 0)
            LAUNCH("row_work", s, k_row_work<<<(unsigned)cdiv(cdiv(A->nnz, 8), 256), 256, 0, s>>>(
                p->a_colptr, p->a_rowidx, K, A->nnz, p->b_rowptr, (unsigned long long *)p->rowwork, p->deg, nullptr));
        TRY(scan_excl(p, p->rowwork, M, p->rowoff, s, "row_offsets"));
        LAUNCH("partition_bounds", s, k_partition_bounds<<<(unsigned)cdiv(parts + 1, 128), 128, 0, s>>>(p->rowoff, M, parts, bounds));
        CK(cudaMemcpyAsync(bounds_host, bounds, (parts + 1) * 8, cudaMemcpyDeviceToHost, s));
        CK(cudaStreamSynchronize(s));
        return SPGEMM_OK;
    }();
    for (void *v : p->owned) cudaFreeAsync(v, s);
    p->owned.clear();
    return r;
}

int spgemm_destroy(spgemm_plan_t p) {
    if (!p) return SPGEMM_OK;
    cudaSetDevice(p->dev);
    for (void *v : p->owned) cudaFreeAsync(v, p->last_stream);
    delete p;
    return SPGEMM_OK;
}

}  // extern "C"
