/*
 * oracle/gustavson.c — CPU ORACLE for the hash-based two-phase CSR SpGEMM
 * (Nagasaka, Nukada, Matsuoka, ICPP 2017; /root/reference/PAPER.md).
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / `--impl reference` leg may load or execute this file.  It shares
 * no code, header, table or constant with the CUDA path
 * (paper_conf_icpp_nagasakanm17_b200/csrc) and neither side includes the other.
 *
 * What it computes (DESIGN.md §3 "Oracle"):
 *   Given CSR A (m x k) and B (k x n), C = A*B with
 *     S(C)  = {(i,j) : exists k with (i,k) in S(A) and (k,j) in S(B)}   (stored patterns;
 *             explicit zeros and cancellations are KEPT — reading R6),
 *     c_ij  = sum_k a_ik * b_kj, each product rounded to and summed in the working
 *             precision (fp32 for SP, fp64 for DP — PAPER.md:179, reading R10),
 *     rows sorted by ascending column, rpt_C[0] = 0.
 *
 * Algorithm: plain row-wise Gustavson (§II-B, Algorithm 1), with the
 * printed if/else read as "insert if c_ij is absent, else accumulate" (reading R1), a
 * dense sparse accumulator of width n (mark/acc), and a per-row qsort.  The two-pass
 * split (count, then fill — PAPER.md:68, 80) only sizes the output; each pass visits
 * products in Algorithm 1's order.
 *
 * Index widths: rpt int64, col int32 (reading R17).  Loop bounds are half-open
 * [rpt[i], rpt[i+1]) (reading R2).  a_rpt[0] need not be 0.
 *
 * Return codes: 0 ok; -1 column index out of range; -2 out of host memory;
 *               -3 numeric row count disagrees with the supplied rpt_C.
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>

/* PAPER.md:90-96 (§III-A, Algorithm 2): n_prod of row i = sum over j in
 * [rpt_A[i], rpt_A[i+1]) of (rpt_B[col_A[j]+1] - rpt_B[col_A[j]]).  Returns the total. */
int64_t oracle_nprod(int64_t m, const int64_t *a_rpt, const int32_t *a_col,
                     const int64_t *b_rpt, int64_t *nprod)
{
    int64_t total = 0;
    for (int64_t i = 0; i < m; ++i) {
        int64_t np = 0;
        for (int64_t j = a_rpt[i]; j < a_rpt[i + 1]; ++j)
            np += b_rpt[a_col[j] + 1] - b_rpt[a_col[j]];
        if (nprod) nprod[i] = np;
        total += np;
    }
    return total;
}

/* First pass of the two-pass strategy: the number of DISTINCT
 * column indices of row i of C (the keys Algorithm 5 would insert),
 * counted with a mark array.  Writes c_rpt[0..m] (exclusive prefix sums). */
int oracle_symbolic(int64_t m, int64_t k, int64_t n,
                    const int64_t *a_rpt, const int32_t *a_col,
                    const int64_t *b_rpt, const int32_t *b_col, int64_t *c_rpt)
{
    int64_t *mark = (int64_t *)malloc((size_t)(n > 0 ? n : 1) * sizeof(int64_t));
    if (!mark) return -2;
    for (int64_t j = 0; j < n; ++j) mark[j] = -1;
    c_rpt[0] = 0;
    for (int64_t i = 0; i < m; ++i) {
        int64_t cnt = 0;
        for (int64_t p = a_rpt[i]; p < a_rpt[i + 1]; ++p) {
            int32_t kk = a_col[p];
            if (kk < 0 || kk >= k) { free(mark); return -1; }
            for (int64_t q = b_rpt[kk]; q < b_rpt[kk + 1]; ++q) {
                int32_t j = b_col[q];
                if (j < 0 || j >= n) { free(mark); return -1; }
                if (mark[j] != i) { mark[j] = i; ++cnt; }
            }
        }
        c_rpt[i + 1] = c_rpt[i] + cnt;
    }
    free(mark);
    return 0;
}

static int cmp_i32(const void *x, const void *y)
{
    int32_t a = *(const int32_t *)x, b = *(const int32_t *)y;
    return (a > b) - (a < b);
}

/* Second pass, Algorithm 1 with a dense accumulator.  VT is the
 * working precision.  c_abs[e] = sum |a_ik|*|b_kj| in double: the scale of the
 * comparison tolerance (DESIGN.md §3 "Comparison rule"), not part of the method. */
#define ORACLE_NUMERIC(NAME, VT)                                                        \
int NAME(int64_t m, int64_t k, int64_t n,                                               \
         const int64_t *a_rpt, const int32_t *a_col, const VT *a_val,                   \
         const int64_t *b_rpt, const int32_t *b_col, const VT *b_val,                   \
         const int64_t *c_rpt, int32_t *c_col, VT *c_val, double *c_abs)                \
{                                                                                       \
    int64_t *mark = (int64_t *)malloc((size_t)(n > 0 ? n : 1) * sizeof(int64_t));       \
    VT *acc = (VT *)malloc((size_t)(n > 0 ? n : 1) * sizeof(VT));                       \
    double *aacc = (double *)malloc((size_t)(n > 0 ? n : 1) * sizeof(double));          \
    if (!mark || !acc || !aacc) { free(mark); free(acc); free(aacc); return -2; }       \
    for (int64_t j = 0; j < n; ++j) mark[j] = -1;                                       \
    for (int64_t i = 0; i < m; ++i) {                                                   \
        int32_t *list = c_col + c_rpt[i]; /* columns of row i in insertion order */     \
        int64_t cnt = 0;                                                                \
        for (int64_t p = a_rpt[i]; p < a_rpt[i + 1]; ++p) {                             \
            int32_t kk = a_col[p];                                                      \
            VT a = a_val[p];                                                            \
            if (kk < 0 || kk >= k) goto bad_index;                                      \
            for (int64_t q = b_rpt[kk]; q < b_rpt[kk + 1]; ++q) {                       \
                int32_t j = b_col[q];                                                   \
                VT value = a * b_val[q];                    /* value <- a_ik b_kj */    \
                double mag = fabs((double)a) * fabs((double)b_val[q]);                  \
                if (j < 0 || j >= n) goto bad_index;                                    \
                if (mark[j] != i) {                         /* c_ij absent: insert */   \
                    if (cnt >= c_rpt[i + 1] - c_rpt[i]) goto bad_count;                 \
                    mark[j] = i; acc[j] = value; aacc[j] = mag; list[cnt++] = j;        \
                } else {                                    /* present: accumulate */   \
                    acc[j] = acc[j] + value; aacc[j] += mag;                            \
                }                                                                       \
            }                                                                           \
        }                                                                               \
        if (cnt != c_rpt[i + 1] - c_rpt[i]) goto bad_count;                             \
        qsort(list, (size_t)cnt, sizeof(int32_t), cmp_i32); /* PAPER.md:173 order */    \
        for (int64_t e = 0; e < cnt; ++e) {                                             \
            c_val[c_rpt[i] + e] = acc[list[e]];                                         \
            if (c_abs) c_abs[c_rpt[i] + e] = aacc[list[e]];                             \
        }                                                                               \
    }                                                                                   \
    free(mark); free(acc); free(aacc);                                                  \
    return 0;                                                                           \
bad_index:                                                                              \
    free(mark); free(acc); free(aacc);                                                  \
    return -1;                                                                          \
bad_count:                                                                              \
    free(mark); free(acc); free(aacc);                                                  \
    return -3;                                                                          \
}

ORACLE_NUMERIC(oracle_numeric_f64, double)
ORACLE_NUMERIC(oracle_numeric_f32, float)

/* ----------------------------------------------------------------------------------------
 * Row-parallel variants: the same two passes for timing the oracle on
 * all host cores and for full-size parity checks (R-MAT s22/s23).  Rows of C are independent
 * (Algorithm 1's outer loop), so each thread runs, for its rows, exactly the loops
 * of oracle_symbolic / Algorithm 1 above on its own dense accumulator: every row is summed in
 * Algorithm 1's product order, and the output is identical to the single-thread functions
 * (tests/test_oracle_pins.py checks that bit for bit).  Compiled with -fopenmp when available;
 * without it they run on one thread.  c_abs may be NULL (no tolerance scale).
 * ---------------------------------------------------------------------------------------- */
#ifdef _OPENMP
#include <omp.h>
#endif

int oracle_threads(void)
{
#ifdef _OPENMP
    return omp_get_max_threads();
#else
    return 1;
#endif
}

/* pass 1: distinct columns per row -> c_rpt (exclusive prefix sums) */
int oracle_symbolic_omp(int64_t m, int64_t k, int64_t n,
                        const int64_t *a_rpt, const int32_t *a_col,
                        const int64_t *b_rpt, const int32_t *b_col, int64_t *c_rpt)
{
    int err = 0;
    c_rpt[0] = 0;
#pragma omp parallel
    {
        int64_t *mark = (int64_t *)malloc((size_t)(n > 0 ? n : 1) * sizeof(int64_t));
        if (!mark) {
#pragma omp atomic write
            err = -2;
        } else {
            for (int64_t j = 0; j < n; ++j) mark[j] = -1;
#pragma omp for schedule(dynamic, 256)
            for (int64_t i = 0; i < m; ++i) {
                int64_t cnt = 0;
                for (int64_t p = a_rpt[i]; p < a_rpt[i + 1]; ++p) {
                    int32_t kk = a_col[p];
                    if (kk < 0 || kk >= k) { err = -1; break; }
                    for (int64_t q = b_rpt[kk]; q < b_rpt[kk + 1]; ++q) {
                        int32_t j = b_col[q];
                        if (j < 0 || j >= n) { err = -1; break; }
                        if (mark[j] != i) { mark[j] = i; ++cnt; }
                    }
                }
                c_rpt[i + 1] = cnt;  /* per-row count; scanned below */
            }
            free(mark);
        }
    }
    if (err) return err;
    for (int64_t i = 0; i < m; ++i) c_rpt[i + 1] += c_rpt[i];
    return 0;
}

#define ORACLE_NUMERIC_OMP(NAME, VT)                                                    \
int NAME(int64_t m, int64_t k, int64_t n,                                               \
         const int64_t *a_rpt, const int32_t *a_col, const VT *a_val,                   \
         const int64_t *b_rpt, const int32_t *b_col, const VT *b_val,                   \
         const int64_t *c_rpt, int32_t *c_col, VT *c_val, double *c_abs)                \
{                                                                                       \
    int err = 0;                                                                        \
    _Pragma("omp parallel")                                                             \
    {                                                                                   \
        int64_t *mark = (int64_t *)malloc((size_t)(n > 0 ? n : 1) * sizeof(int64_t));   \
        VT *acc = (VT *)malloc((size_t)(n > 0 ? n : 1) * sizeof(VT));                   \
        double *aacc = c_abs ? (double *)malloc((size_t)(n > 0 ? n : 1) * sizeof(double)) \
                             : NULL;                                                    \
        if (!mark || !acc || (c_abs && !aacc)) {                                        \
            err = -2;                                                                   \
        } else {                                                                        \
            for (int64_t j = 0; j < n; ++j) mark[j] = -1;                               \
            _Pragma("omp for schedule(dynamic, 256)")                                   \
            for (int64_t i = 0; i < m; ++i) {                                           \
                int32_t *list = c_col + c_rpt[i];                                       \
                int64_t cnt = 0, cap = c_rpt[i + 1] - c_rpt[i];                          \
                for (int64_t p = a_rpt[i]; p < a_rpt[i + 1] && !err; ++p) {             \
                    int32_t kk = a_col[p];                                              \
                    VT a = a_val[p];                                                    \
                    if (kk < 0 || kk >= k) { err = -1; break; }                         \
                    for (int64_t q = b_rpt[kk]; q < b_rpt[kk + 1]; ++q) {               \
                        int32_t j = b_col[q];                                           \
                        VT value = a * b_val[q];                /* value <- a_ik b_kj */ \
                        if (j < 0 || j >= n) { err = -1; break; }                       \
                        if (mark[j] != i) {                     /* absent: insert */    \
                            if (cnt >= cap) { err = -3; break; }                        \
                            mark[j] = i; acc[j] = value; list[cnt++] = j;               \
                            if (aacc) aacc[j] = fabs((double)a) * fabs((double)b_val[q]); \
                        } else {                                /* present: accumulate */ \
                            acc[j] = acc[j] + value;                                    \
                            if (aacc) aacc[j] += fabs((double)a) * fabs((double)b_val[q]); \
                        }                                                               \
                    }                                                                   \
                }                                                                       \
                if (err) continue;                                                      \
                if (cnt != cap) { err = -3; continue; }                                 \
                qsort(list, (size_t)cnt, sizeof(int32_t), cmp_i32);                     \
                for (int64_t e = 0; e < cnt; ++e) {                                     \
                    c_val[c_rpt[i] + e] = acc[list[e]];                                 \
                    if (aacc) c_abs[c_rpt[i] + e] = aacc[list[e]];                      \
                }                                                                       \
            }                                                                           \
        }                                                                               \
        free(mark); free(acc); free(aacc);                                              \
    }                                                                                   \
    return err;                                                                         \
}

ORACLE_NUMERIC_OMP(oracle_numeric_omp_f64, double)
ORACLE_NUMERIC_OMP(oracle_numeric_omp_f32, float)
