/*
 * spgemm.h -- C-ABI of the B200 outer-product spGEMM with the Block Reorganizer.
 *
 * Problem (§II-B, reconstructed Eq. (2); §IV):
 *     C = A x B = sum_k  a_*k (outer) b_k*
 * A (m x k) is consumed by columns (CSC, "a_*k"), B (k x n) by rows (CSR, "b_k*"),
 * exactly the A'ptr/A'idx/A'val and B'ptr/B'idx/B'val arrays of Fig. 5 (L333-L339).
 * C is returned as canonical CSR: int64 row pointers, int32 column indices sorted
 * ascending within each row, fp32 values; every (i,j) that received at least one
 * product is stored, including computed zeros (reading R7).
 *
 * Pipeline behind the calls (DESIGN.md §1, §8 rows):
 *   spgemm_plan     (1) workload analysis: block-wise nnz(a_*k)*nnz(b_k*) and row-wise
 *                       nnz of Ĉ (L326-L330 L, L289-L291 R), Ĉ row offsets and run bases;
 *                   (2) categorisation (Dominator / Normal / Low performer, L304-L318 R),
 *                       B-Splitting pieces (L320-L415), B-Gathering lists (L369-L450),
 *                       merge row bins incl. B-Limiting rows (L452-L477 L).
 *   spgemm_expand   (3) expansion: every product (i, j, a_ik*b_kj) written into the
 *                       row-bucketed intermediate matrix Ĉ (L321-L323 L).
 *   spgemm_merge    (4) merge: per Ĉ row, sort by column + segmented reduce (fp64
 *                       accumulation, one rounding to fp32); long rows B-Limited.  Rows are
 *                       merged in place in their Ĉ buckets (default), or -- tile merge,
 *                       options.reserved[5] = 2 -- placed by a decoupled look-back at the head
 *                       of the Ĉ arrays (C in place, no compaction pass).
 *   spgemm_output       CSR compaction of the merged rows into caller buffers (tile merge: a copy
 *                       of C's head, nothing when the caller's arrays are the Ĉ arrays).
 *   spgemm_execute  = expand + merge + allocate C (callback) + output.
 *
 * Conventions for every call:
 *   - return value: SPGEMM_OK (0) or a spgemm_status error code; on error a
 *     human-readable reason is available from spgemm_last_error() (thread-local).
 *   - `stream` is a cudaStream_t (NULL = legacy default stream).  All device work is
 *     ordered on it.  Calls that must return host-side sizes synchronise it.
 *   - Pointers in matrix descriptors are device pointers when `where` is
 *     SPGEMM_DEVICE and host pointers when SPGEMM_HOST (host inputs are copied to the
 *     device inside spgemm_plan; pinned host memory makes those copies asynchronous).
 *   - The caller keeps ownership of A and B; device inputs must stay valid and
 *     unmodified until spgemm_destroy.  The plan owns its workspaces.
 *   - Requirements (checked when options.validate != 0, else undefined behaviour):
 *     ptr arrays non-decreasing with ptr[0] = 0 and ptr[last] = nnz; indices in range
 *     and strictly increasing within each column of A / row of B; A.ncols == B.nrows;
 *     dimensions < 2^31.
 *   - A plan is single-use and not thread-safe; it binds to the current CUDA device
 *     at spgemm_plan time.
 */
#ifndef SPGEMM_H
#define SPGEMM_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define SPGEMM_ABI_VERSION 1

typedef enum {
    SPGEMM_OK = 0,
    SPGEMM_ERR_INVALID_ARGUMENT = 1, /* NULL pointer, bad dimension, bad option           */
    SPGEMM_ERR_INVALID_INPUT = 2,    /* validate: malformed CSC/CSR (unsorted, range)      */
    SPGEMM_ERR_CUDA = 3,             /* a CUDA runtime error (message in last_error)       */
    SPGEMM_ERR_OUT_OF_MEMORY = 4,    /* device or host allocation failed                    */
    SPGEMM_ERR_STATE = 5,            /* calls out of order (e.g. merge before expand)       */
    SPGEMM_ERR_NO_DEVICE = 6         /* no CUDA device / library built for another arch    */
} spgemm_status;

typedef enum { SPGEMM_DEVICE = 0, SPGEMM_HOST = 1 } spgemm_where;

/* A (m x k), compressed sparse column.  colptr[ncols+1] int64, rowidx[nnz] int32
 * ascending within each column, val[nnz] fp32. */
typedef struct {
    int64_t nrows, ncols, nnz;
    const int64_t *colptr;
    const int32_t *rowidx;
    const float *val;
    int32_t where; /* spgemm_where */
} spgemm_csc_t;

/* B (k x n), compressed sparse row.  rowptr[nrows+1] int64, colidx[nnz] int32 ascending
 * within each row, val[nnz] fp32. */
typedef struct {
    int64_t nrows, ncols, nnz;
    const int64_t *rowptr;
    const int32_t *colidx;
    const float *val;
    int32_t where;
} spgemm_csr_t;

/* C (m x n) output, canonical CSR.  Filled by spgemm_output / spgemm_execute. */
typedef struct {
    int64_t nrows, ncols, nnz;
    int64_t *rowptr; /* [nrows+1] */
    int32_t *colidx; /* [nnz]     */
    float *val;      /* [nnz]     */
    int32_t where;
} spgemm_csr_out_t;

/* Tunables.  Call spgemm_default_options() first; zero keeps a B200-derived default.
 * Paper parameters keep the paper's names (α, β); DESIGN.md §2 R1-R8 gives the readings. */
typedef struct {
    double alpha;             /* >0: Dominator threshold nnz(Ĉ)/(#pair blocks × α) (L309-L311 R);
                                 0: B200 default clamp(nnz(Ĉ)/(#SMs × dom_waves),
                                    dom_min_work, piece_work)                                   */
    int32_t dom_waves;        /* B200 default: fair-share divisor per SM (default 16)           */
    int64_t dom_min_work;     /* lower bound of the B200 Dominator threshold (default 4096)     */
    int32_t split_ca_max;     /* max computations per thread nnz(a_*k) of a piece (default 256) */
    int64_t piece_work;       /* max products of one B-Splitting piece (default 16384)          */
    int32_t split_b_tile;     /* max B-row entries per piece (default 4096)                     */
    double beta;              /* >0: limiting threshold min(cap, nnz(Ĉ)/(#rows × β)) (L475-L477 L);
                                 0: B200 default = non-limited merge capacity (4096)            */
    int32_t limit_ctas_per_sm;/* B-Limiting (PAPER.md L463-L469 L, Fig. 14): resident limited-
                                 merge blocks per SM, 1 / 2 / 4 = blocks of 1024 / 512 / 256
                                 threads sorting column groups of <= 9216 / 4096 / 2048
                                 products (other values round down to these; default 1).  With
                                 2 or 4, rows with a column range too heavy for the smaller
                                 sorter are deferred to a second launch at 1 per SM.        */
    int32_t enable_split;     /* ablation switches (Fig. 10): 0 disables the technique; for
                                 enable_limit = 0 the β threshold is ignored and only rows above
                                 the non-limited kernels' capacity take the long-row kernels     */
    int32_t enable_gather;
    int32_t enable_limit;
    int32_t validate;         /* check input structure in spgemm_plan (default 1).  With 0 the
                                 caller guarantees the contracts above: the merge relies on B's
                                 ascending rows (each run is sorted; the per-row column range is
                                 read from the first / last entry of b_k*) -- unsorted rows are
                                 then undefined behaviour, not an error                          */
    int32_t reserved[16];     /* tuning / comparison knobs, 0 = default:
                                 [0] unused (round-1 merge variants, removed in round 2);
                                 [1] profiling: 1 tile merge without look-back (wrong C, timing
                                     only), 2 tile-merge phase clocks, 3 B-Limited path clocks
                                     (SPGEMM_VIEW_UNIT_PROFILE);
                                 [2] 1 = per-row compaction kernels instead of the chunked one;
                                 [3] 1 = row-product expansion (the paper's comparison order);
                                 [4] 1 = no per-row column range from the plan (the merge
                                     reduces each row's min / max column itself);
                                 [5] 2 = tile merge (merge_tiles.cuh, merge_long.cuh): tiles of
                                     short rows and column groups of the long rows in row order,
                                     C placed by look-back in place, no compaction ([0] = 0);
                                 [6] 1 = with [5] = 2: long rows by the per-bin long-row kernels
                                     (merged in place, then moved) instead of column groups;
                                 [7] > 0: fixed B-Splitting factor for every Dominator (the
                                     Fig. 11 sweep; capped at the column's power of two);
                                 [8] 1 = record per-SM busy times for the LBI (SPGEMM_VIEW_LBI);
                                 [9] expansion mapping: 0 block path (split pieces + Normal blocks,
                                     TMA-staged) + a 16-byte vector per thread for the gathered
                                     Low performers, 1 every block a vector per thread (round 1);
                                 [11] 1 = rows of 33-256 slots by the warp merge path (round 1)
                                     instead of a warp-per-row bucket sort (64 / 128 / 256 slots) */
} spgemm_options_t;

/* Sizes and bin populations of a plan (spgemm_get_stats). */
typedef struct {
    int64_t m, k, n, nnz_a, nnz_b;
    int64_t nnz_chat;          /* intermediate products = sum_k nnz(a_*k) nnz(b_k*)            */
    int64_t nnz_chat_rowwise;  /* the same count, summed row-wise (must equal nnz_chat)       */
    int64_t nnz_c;             /* after spgemm_merge, else -1                                  */
    int64_t k_nonempty, m_nonempty;
    int64_t t_dom, t_lim;      /* thresholds actually used                                     */
    int64_t n_dominator, n_normal, n_low, n_pieces_split;
    int64_t n_gather_bin[6];   /* low performers per gathering bin n (2^(n-1) < t <= 2^n)      */
    int64_t n_rows_bin[6];     /* empty, single-run, <=32 slots, <=1024 slots, <=4096 slots, limited */
    int64_t bytes_workspace;   /* device bytes held by the plan                                */
    int64_t n_units;           /* tile merge: tiles walked (after spgemm_merge), else -1          */
    int64_t n_units_fallback;  /* tile merge: 0 (no fallback path), else -1                    */
} spgemm_stats_t;

/* spgemm_inspect selectors: copy a plan array to host memory (tests, tooling). */
typedef enum {
    SPGEMM_VIEW_WORK = 0,        /* int64[k]   block-wise work nnz(a_*k)*nnz(b_k*)          */
    SPGEMM_VIEW_ROWWORK = 1,     /* int64[m]   row-wise nnz of Ĉ                             */
    SPGEMM_VIEW_ROWOFF = 2,      /* int64[m+1] Ĉ row offsets                                 */
    SPGEMM_VIEW_PAIR_CLASS = 3,  /* int8[k]    0 empty, 1 dominator, 2 normal, 3 low         */
    SPGEMM_VIEW_PIECES = 4,      /* int64[n_pieces_split][5] (k, a_lo, a_hi, b_lo, b_hi)     */
    SPGEMM_VIEW_GATHER = 5,      /* int32[n_low] pairs in packing order, bins n = 0..5 in turn */
    SPGEMM_VIEW_ROW_CLASS = 6,   /* int8[m]    0 empty, 1 passthrough, 2 warp, 3 warp-radix,
                                                4 cta-radix, 5 limited                        */
    SPGEMM_VIEW_CHAT_COL = 7,    /* int32[nnz_chat] after spgemm_expand (before merge)       */
    SPGEMM_VIEW_CHAT_VAL = 8,    /* fp32[nnz_chat]                                            */
    SPGEMM_VIEW_CROWPTR = 9,     /* int64[m+1] C row pointers after spgemm_merge             */
    SPGEMM_VIEW_UNIT_PROFILE = 10,/* uint64[16] merge phase clocks (options.reserved[1] = 2 / 3)  */
    SPGEMM_VIEW_ROW_COLMIN = 11, /* int32[m]   first column of row i of C (the merge's bucket
                                    range; computed in spgemm_plan for rows whose padded Ĉ
                                    bucket exceeds 256 slots; other rows 0x7f7f7f7f = unknown;
                                    size 0 with options.reserved[4] = 1)                       */
    SPGEMM_VIEW_ROW_COLMAX = 12, /* int32[m]   last column of row i of C (unknown rows 0)     */
    SPGEMM_VIEW_LBI = 13         /* uint64[2][257] with options.reserved[8] = 1, after the kernels ran:
                                    per kernel (0 expansion, 1 B-Limited merge) [0] = first CTA start,
                                    [1 + smid] = last CTA end on that SM (%globaltimer ns); the
                                    load balancing index of PAPER.md Eq. (3) (L564-L577 R) is
                                    mean_i(T_i) / max_i(T_i), T_i = [1 + i] - [0] over the SMs     */
} spgemm_view;

typedef struct spgemm_plan_s *spgemm_plan_t;

/* Allocator used by spgemm_execute for C: returns `bytes` of memory in `where`
 * (SPGEMM_DEVICE or SPGEMM_HOST), or NULL on failure.  The caller owns the memory. */
typedef void *(*spgemm_alloc_fn)(size_t bytes, int32_t where, void *ctx);

int spgemm_abi_version(void);
const char *spgemm_last_error(void);
void spgemm_default_options(spgemm_options_t *opt);

/* Stages (1)+(2).  Synchronises `stream` twice (to size Ĉ and the bins).  On success
 * *plan is a new plan; on failure *plan is NULL and nothing is leaked. */
int spgemm_plan(const spgemm_csc_t *A, const spgemm_csr_t *B, const spgemm_options_t *opt,
                void *stream, spgemm_plan_t *plan);

/* Rows [row_begin, row_end) of C = A x B, planned without a copy of A by the caller: the window's
 * entries of every column of A (one contiguous range, rows being ascending) are packed on the
 * device into the plan's own A' (row indices minus row_begin), so the plan computes the
 * (row_end - row_begin) x n row block of C (the chunked expansion and the multi-GPU row blocks of
 * DESIGN.md R8).  Synchronises `stream` once more than spgemm_plan (the window's nnz).
 * spgemm_plan(A, B, ...) = spgemm_plan_rows(A, B, 0, A->nrows, ...). */
int spgemm_plan_rows(const spgemm_csc_t *A, const spgemm_csr_t *B, int64_t row_begin, int64_t row_end,
                     const spgemm_options_t *opt, void *stream, spgemm_plan_t *plan);

/* Stage (3): writes Ĉ.  Asynchronous. */
int spgemm_expand(spgemm_plan_t plan, void *stream);

/* Stage (4): merges Ĉ in place and scans the row counts; returns nnz(C) in *nnz_c
 * (synchronises `stream`). */
int spgemm_merge(spgemm_plan_t plan, void *stream, int64_t *nnz_c);

/* Compaction into caller-provided C arrays (C->where chooses device or host; sizes
 * nrows+1 / nnz(C) / nnz(C)).  Asynchronous for device outputs; host outputs
 * synchronise `stream` before returning. */
int spgemm_output(spgemm_plan_t plan, spgemm_csr_out_t *C, void *stream);

/* expand + merge + alloc(C arrays in `out_where`) + output.  C->rowptr/colidx/val are
 * set to the allocated buffers (owned by the caller).  Returns after `stream` holds C.
 * With a device C and the tile merge (options.reserved[5] = 2),
 * colidx / val are requested BEFORE the expansion with capacity nnz(Ĉ) (padded slots) >= nnz(C):
 * they hold Ĉ during the merge and C in their first C->nnz entries afterwards (one buffer for
 * both: no second nnz(Ĉ)-sized allocation, no copy). */
int spgemm_execute(spgemm_plan_t plan, spgemm_alloc_fn alloc, void *alloc_ctx, int32_t out_where,
                   spgemm_csr_out_t *C, void *stream);

int spgemm_get_stats(spgemm_plan_t plan, spgemm_stats_t *stats);

/* Copies view `what` into host_dst (capacity bytes); *size_bytes receives the full size.
 * Synchronises the device.  Returns SPGEMM_ERR_INVALID_ARGUMENT if capacity is short. */
int spgemm_inspect(spgemm_plan_t plan, int32_t what, void *host_dst, int64_t capacity_bytes,
                   int64_t *size_bytes);

/* Frees every workspace of the plan (stream-ordered on the plan's last stream).  Workspaces
 * include the temporaries of every call (e.g. host-output staging): they live until here. */
int spgemm_destroy(spgemm_plan_t plan);

/* Multi-GPU / chunked execution: balanced row-block partition of C = A x B (R8).
 * Computes the row-wise nnz of Ĉ on the device and returns in bounds_host[parts+1] the row
 * boundaries r_0 = 0 <= ... <= r_parts = m, r_p = first row whose Ĉ prefix reaches
 * floor(p * nnz(Ĉ) / parts).  Synchronises `stream`.  Inputs as for spgemm_plan. */
int spgemm_row_partition(const spgemm_csc_t *A, const spgemm_csr_t *B, int32_t parts, int64_t *bounds_host,
                         void *stream);

/* Plans allocate their workspaces from a per-device stream-ordered pool that keeps freed memory
 * for the next plan (no OS allocation per step).  spgemm_trim_pool returns the current device's
 * cached memory to the driver (e.g. before allocating a large C or between very large products).
 * Synchronises the device. */
int spgemm_trim_pool(void);

/* Per-kernel device timing of the last spgemm_expand / spgemm_merge (CUDA events on the
 * launch stream; enabled by spgemm_set_timing(1)).  names/ms arrays of capacity n. */
int spgemm_set_timing(int32_t enable);
int spgemm_last_timings(const char **names, float *ms, int32_t capacity, int32_t *count);

#ifdef __cplusplus
}
#endif

#endif /* SPGEMM_H */
