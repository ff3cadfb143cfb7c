/*
 * synth/rmat.c — seeded R-MAT graph generator (BASELINE.json config 5; SURVEY.md §8(d) recipe),
 * INPUT GENERATION ONLY: no SpGEMM arithmetic (no products, counts of products, hashing or
 * binning).  Shared by the oracle tests, the CUDA parity tests and bench.py through
 * synth/matrices.py (ctypes), compiled with gcc -O3 -fopenmp on first use.
 *
 * Recipe: N = 2^scale vertices, E = ef * N directed edges.  For edge e and level l < scale one
 * uniform u in [0,1) is drawn; row bit l = [u >= a+b], column bit l = [a <= u < a+b] or
 * [u >= a+b+c].  Duplicate edges are merged, columns sorted, no relabelling (hubs at low indices).
 *
 * Random numbers: a counter-based generator, so any subset of edges can be drawn independently
 * and in parallel with an identical result: x = mix64(mix64(seed) ^ (e * 64 + l)) with mix64 the
 * splitmix64 finaliser, u = (x >> 11) * 2^-53.  synth/matrices.py:_rmat_numpy implements the same
 * draw in NumPy for small scales (tests/test_synth.py compares the two CSR outputs exactly).
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

static inline uint64_t mix64(uint64_t z)
{
    z += 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}

static int cmp_i32(const void *x, const void *y)
{
    int32_t a = *(const int32_t *)x, b = *(const int32_t *)y;
    return (a > b) - (a < b);
}

static void sort_row(int32_t *v, int64_t n)
{
    if (n > 24) { qsort(v, (size_t)n, sizeof(int32_t), cmp_i32); return; }
    for (int64_t i = 1; i < n; ++i) {  /* insertion sort for the (typical) short rows */
        int32_t x = v[i];
        int64_t j = i - 1;
        while (j >= 0 && v[j] > x) { v[j + 1] = v[j]; --j; }
        v[j + 1] = x;
    }
}

/* rpt: int64[N+1] (caller); col: int32[ef*N] (caller, upper bound); returns nnz after merging
 * duplicates (col[0..nnz) valid), or -1 on allocation failure. */
int64_t rmat_csr(int scale, int64_t ef, double a, double b, double c, uint64_t seed,
                 int64_t *rpt, int32_t *col)
{
    const int64_t N = (int64_t)1 << scale, E = ef * N;
    const double ab = a + b, abc = a + b + c;
    const uint64_t s0 = mix64(seed);
    int32_t *er = (int32_t *)malloc((size_t)E * sizeof(int32_t));
    int32_t *ec = (int32_t *)malloc((size_t)E * sizeof(int32_t));
    int64_t *cnt = (int64_t *)calloc((size_t)N + 1, sizeof(int64_t));
    int64_t *uniq = (int64_t *)calloc((size_t)N + 1, sizeof(int64_t));
    int32_t *tmp = (int32_t *)malloc((size_t)E * sizeof(int32_t));
    if (!er || !ec || !cnt || !uniq || !tmp) {
        free(er); free(ec); free(cnt); free(uniq); free(tmp);
        return -1;
    }
    /* 1. edges */
#pragma omp parallel for schedule(static)
    for (int64_t e = 0; e < E; ++e) {
        int64_t r = 0, q = 0;
        for (int l = 0; l < scale; ++l) {
            const double u = (double)(mix64(s0 ^ ((uint64_t)e * 64u + (uint64_t)l)) >> 11) * 0x1.0p-53;
            r |= (int64_t)(u >= ab) << l;
            q |= (int64_t)((u >= a && u < ab) || u >= abc) << l;
        }
        er[e] = (int32_t)r;
        ec[e] = (int32_t)q;
        __atomic_fetch_add(&cnt[r + 1], 1, __ATOMIC_RELAXED);
    }
    /* 2. bucket the edges by row (order inside a row is fixed by the sort below) */
    for (int64_t i = 0; i < N; ++i) cnt[i + 1] += cnt[i];
    int64_t *cur = uniq;  /* reused as the scatter cursor, reset below */
    memcpy(cur, cnt, (size_t)N * sizeof(int64_t));
#pragma omp parallel for schedule(static)
    for (int64_t e = 0; e < E; ++e) {
        const int64_t p = __atomic_fetch_add(&cur[er[e]], 1, __ATOMIC_RELAXED);
        tmp[p] = ec[e];
    }
    free(er);
    free(ec);
    /* 3. sort + merge duplicates per row */
#pragma omp parallel for schedule(dynamic, 4096)
    for (int64_t i = 0; i < N; ++i) {
        int32_t *v = tmp + cnt[i];
        const int64_t n = cnt[i + 1] - cnt[i];
        sort_row(v, n);
        int64_t u = 0;
        for (int64_t j = 0; j < n; ++j)
            if (u == 0 || v[j] != v[u - 1]) v[u++] = v[j];
        uniq[i] = u;
    }
    rpt[0] = 0;
    for (int64_t i = 0; i < N; ++i) rpt[i + 1] = rpt[i] + uniq[i];
#pragma omp parallel for schedule(dynamic, 4096)
    for (int64_t i = 0; i < N; ++i)
        memcpy(col + rpt[i], tmp + cnt[i], (size_t)(rpt[i + 1] - rpt[i]) * sizeof(int32_t));
    const int64_t nnz = rpt[N];
    free(cnt);
    free(uniq);
    free(tmp);
    return nnz;
}
