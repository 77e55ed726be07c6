/*
 * ORACLE -- TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and
 * bench.py's cpu_baseline / --impl reference leg may load this library.  It
 * shares no code with the CUDA path (paper_conf_icde_leekyjkp20_b200/csrc).
 *
 * Plain, slow, obviously-correct CPU spGEMM C = A x B by the row product
 * (Gustavson [19]; PAPER.md L199-L211 R "Gustavson's dense accumulator ...
 * a temporary array with a length equal to the dimension of the target matrix",
 * and the paper's row-product baseline L476-L478 R):
 *
 *     c_i* = sum_k a_ik * b_k*                         (reconstructed Eq. (1))
 *
 * accumulated in fp64 in a dense accumulator of length n, with a "touched"
 * flag per column so that computed zeros are kept in the structure (an entry
 * (i,j) exists iff at least one product a_ik*b_kj was formed).  Columns of
 * each output row are emitted in ascending order (canonical CSR).
 *
 * Inputs follow the library's boundary layout: A (m x k) CSC with int64
 * colptr / int32 rowidx / f32 val, B (k x n) CSR with int64 rowptr / int32
 * colidx / f32 val.  The oracle first transposes A to CSR (counting
 * transpose), then runs the textbook row loop.  OpenMP parallelises the
 * independent rows only; each row is computed exactly as the serial loop.
 *
 * Optional row subset: rows[] lists the output rows to compute (used to check
 * full-size runs on a sample of rows, one by one).
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

/* A (CSC) -> A (CSR): at_rowptr[m+1], at_colidx[nnz], at_val[nnz]. */
static int transpose_csc_to_csr(int64_t m, int64_t k, const int64_t *colptr, const int32_t *rowidx,
                                const float *val, int64_t **o_ptr, int32_t **o_idx, float **o_val) {
    int64_t nnz = colptr[k];
    int64_t *ptr = (int64_t *)calloc((size_t)m + 1, sizeof(int64_t));
    int32_t *idx = (int32_t *)malloc((size_t)(nnz > 0 ? nnz : 1) * sizeof(int32_t));
    float *v = (float *)malloc((size_t)(nnz > 0 ? nnz : 1) * sizeof(float));
    int64_t *cur = (int64_t *)malloc(((size_t)m + 1) * sizeof(int64_t));
    if (!ptr || !idx || !v || !cur) { free(ptr); free(idx); free(v); free(cur); return -1; }
    for (int64_t e = 0; e < nnz; ++e) ptr[rowidx[e] + 1] += 1;
    for (int64_t i = 0; i < m; ++i) ptr[i + 1] += ptr[i];
    memcpy(cur, ptr, ((size_t)m + 1) * sizeof(int64_t));
    for (int64_t c = 0; c < k; ++c)               /* columns in ascending order, so    */
        for (int64_t e = colptr[c]; e < colptr[c + 1]; ++e) {  /* each row's list is */
            int64_t p = cur[rowidx[e]]++;                        /* ascending in k    */
            idx[p] = (int32_t)c;
            v[p] = val[e];
        }
    free(cur);
    *o_ptr = ptr; *o_idx = idx; *o_val = v;
    return 0;
}

static int cmp_i32(const void *a, const void *b) {
    int32_t x = *(const int32_t *)a, y = *(const int32_t *)b;
    return (x > y) - (x < y);
}

/*
 * Pass 1 (symbolic): count[r] = |{ j : exists k, a_ik != 0 (stored) and b_kj stored }|
 * for each requested row i = rows[r] (or i = r when rows == NULL).
 * Pass 2 (numeric): fills col/val of the rows at out_ptr[r] .. out_ptr[r+1].
 * Both passes use the same row routine; fill == 0 only counts.
 */
static int64_t gustavson_row(int64_t i, const int64_t *at_ptr, const int32_t *at_idx, const float *at_val,
                             const int64_t *b_rowptr, const int32_t *b_colidx, const float *b_val,
                             double *acc, unsigned char *touched, int32_t *list,
                             int fill, int32_t *out_col, double *out_val) {
    int64_t cnt = 0;
    for (int64_t p = at_ptr[i]; p < at_ptr[i + 1]; ++p) {
        int32_t kk = at_idx[p];
        double a = (double)at_val[p];
        for (int64_t q = b_rowptr[kk]; q < b_rowptr[kk + 1]; ++q) {
            int32_t j = b_colidx[q];
            if (!touched[j]) { touched[j] = 1; acc[j] = 0.0; list[cnt++] = j; }
            acc[j] += a * (double)b_val[q];
        }
    }
    qsort(list, (size_t)cnt, sizeof(int32_t), cmp_i32);
    for (int64_t t = 0; t < cnt; ++t) {
        int32_t j = list[t];
        if (fill) { out_col[t] = j; out_val[t] = acc[j]; }
        touched[j] = 0;
    }
    return cnt;
}

static int run(int64_t m, int64_t k, int64_t n,
               const int64_t *a_colptr, const int32_t *a_rowidx, const float *a_val,
               const int64_t *b_rowptr, const int32_t *b_colidx, const float *b_val,
               const int32_t *rows, int64_t nrows, int fill,
               int64_t *out_count, const int64_t *out_ptr, int32_t *out_col, double *out_val,
               int nthreads) {
    int64_t *at_ptr; int32_t *at_idx; float *at_val;
    if (transpose_csc_to_csr(m, k, a_colptr, a_rowidx, a_val, &at_ptr, &at_idx, &at_val)) return -1;
    int err = 0;
#ifdef _OPENMP
    if (nthreads > 0) omp_set_num_threads(nthreads);
#else
    (void)nthreads;
#endif
#pragma omp parallel
    {
        double *acc = (double *)malloc((size_t)(n > 0 ? n : 1) * sizeof(double));
        unsigned char *touched = (unsigned char *)calloc((size_t)(n > 0 ? n : 1), 1);
        int32_t *list = (int32_t *)malloc((size_t)(n > 0 ? n : 1) * sizeof(int32_t));
        if (!acc || !touched || !list) {
#pragma omp atomic write
            err = 1;
        } else {
#pragma omp for schedule(dynamic, 64)
            for (int64_t r = 0; r < nrows; ++r) {
                int64_t i = rows ? (int64_t)rows[r] : r;
                int64_t c = gustavson_row(i, at_ptr, at_idx, at_val, b_rowptr, b_colidx, b_val, acc, touched,
                                          list, fill, fill ? out_col + out_ptr[r] : NULL,
                                          fill ? out_val + out_ptr[r] : NULL);
                if (out_count) out_count[r] = c;
            }
        }
        free(acc); free(touched); free(list);
    }
    free(at_ptr); free(at_idx); free(at_val);
    return err ? -1 : 0;
}

/* Row counts of C (symbolic).  rows == NULL means all m rows (nrows must equal m). */
int oracle_gustavson_count(int64_t m, int64_t k, int64_t n,
                           const int64_t *a_colptr, const int32_t *a_rowidx, const float *a_val,
                           const int64_t *b_rowptr, const int32_t *b_colidx, const float *b_val,
                           const int32_t *rows, int64_t nrows, int64_t *out_count, int nthreads) {
    return run(m, k, n, a_colptr, a_rowidx, a_val, b_rowptr, b_colidx, b_val, rows, nrows, 0,
               out_count, NULL, NULL, NULL, nthreads);
}

/* Numeric fill of the rows, at offsets out_ptr[r] (exclusive scan of the counts). */
int oracle_gustavson_fill(int64_t m, int64_t k, int64_t n,
                          const int64_t *a_colptr, const int32_t *a_rowidx, const float *a_val,
                          const int64_t *b_rowptr, const int32_t *b_colidx, const float *b_val,
                          const int32_t *rows, int64_t nrows, const int64_t *out_ptr,
                          int32_t *out_col, double *out_val, int nthreads) {
    return run(m, k, n, a_colptr, a_rowidx, a_val, b_rowptr, b_colidx, b_val, rows, nrows, 1,
               NULL, out_ptr, out_col, out_val, nthreads);
}

int oracle_max_threads(void) {
#ifdef _OPENMP
    return omp_get_max_threads();
#else
    return 1;
#endif
}
