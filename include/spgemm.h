/*
 * spgemm.h — C ABI of the B200-native (sm_100a) hash-based two-phase CSR SpGEMM
 *            C = A * B  (Nagasaka, Nukada, Matsuoka, ICPP 2017; /root/reference/PAPER.md).
 *
 * Library: paper_conf_icpp_nagasakanm17_b200/libspgemm.so.  extern "C", plain pointers and
 * sizes only; no CUDA or torch types appear in a signature (streams are passed as the
 * opaque value of a cudaStream_t, `void*`).  Pointers are DEVICE pointers unless marked
 * (host).
 *
 * Problem statement: A (m x k) and B (k x n) and C are CSR; the
 * pattern of C is unknown until computed, so a counting ("symbolic") pass sizes C exactly
 * before a calculation ("numeric") pass fills it — the two-pass strategy of PAPER.md:68
 * that "does not require redundant working memory".
 *
 * CSR layout: row i of X is col[rpt[i] .. rpt[i+1]) with values at the same
 * offsets.  rpt is int64 (nnz(C) exceeds 2^31 at R-MAT scale 22 — DESIGN.md reading R17),
 * col is int32, 0 <= col < n <= 2^31-2 (the key -1 is the empty-slot marker of
 * Algorithm 5).  a_rpt[0] need NOT be 0 (zero-copy row slices).
 * Input rows need not be sorted; duplicate column indices behave as their sum.  Explicit
 * zeros and cancellations are kept structurally (reading R6).  Output rows are sorted by
 * ascending column.
 *
 * Ownership: the caller owns A, B and all of C.  The library owns only its workspace
 * (grouping arrays, n_prod, global-memory hash tables), obtained from the allocator given to
 * spgemm_create (NULL -> a private stream-ordered CUDA memory pool of the handle whose
 * memory stays mapped between calls and is released by spgemm_destroy).  Workspace buffers
 * are grow-only: kept across calls (stable addresses for graph replay) until spgemm_destroy.  A's and B's structure
 * arrays are BORROWED from spgemm_symbolic until the next spgemm_symbolic/destroy: they
 * must stay alive and unchanged while spgemm_numeric may be called (structure reuse).
 *
 * Ordering: all work is enqueued on the handle's stream (plus internal streams forked from
 * and joined back into it).  spgemm_symbolic returns after synchronising that stream (the
 * host needs nnz(C) to allocate C — PAPER.md:80, 282).  spgemm_numeric is asynchronous.
 * A handle is not thread-safe: one handle per host thread / stream.
 *
 * Errors: status codes only; no C++ exception crosses the ABI.  Detailed text via
 * spgemm_last_error(h).  Any CUDA failure returns SPGEMM_ERR_CUDA.
 */
#ifndef SPGEMM_H_
#define SPGEMM_H_

#include <stddef.h>
#include <stdint.h>

#if defined(__GNUC__)
#define SPGEMM_API __attribute__((visibility("default")))
#else
#define SPGEMM_API
#endif

#ifdef __cplusplus
extern "C" {
#endif

typedef struct spgemm_ctx *spgemm_handle_t;

typedef enum { SPGEMM_F32 = 0, SPGEMM_F64 = 1 } spgemm_dtype_t;

typedef enum {
    SPGEMM_OK = 0,
    SPGEMM_ERR_INVALID_ARG = 1,     /* NULL pointer, negative size, bad enum */
    SPGEMM_ERR_BAD_STATE = 2,       /* numeric before symbolic, etc. */
    SPGEMM_ERR_OOM = 3,             /* allocator returned NULL */
    SPGEMM_ERR_CUDA = 4,            /* CUDA runtime error; text in spgemm_last_error */
    SPGEMM_ERR_INDEX_OVERFLOW = 5,  /* n > 2^31-2 or m >= 2^31 */
    SPGEMM_ERR_NOT_SUPPORTED = 6,   /* device is not sm_100 */
    SPGEMM_ERR_INVALID_INPUT = 7    /* validation on: rpt not monotone or col out of range */
} spgemm_status_t;

/* Stream-ordered allocator callbacks.  alloc returns NULL on failure. */
typedef struct {
    void *(*alloc)(size_t bytes, void *stream, void *ctx);
    void (*free)(void *ptr, size_t bytes, void *stream, void *ctx);
    void *ctx;
} spgemm_allocator_t;

/* Create a handle on CUDA device `device`, enqueueing on `stream` (a cudaStream_t; NULL =
 * legacy default stream).  alloc may be NULL.  Fails with NOT_SUPPORTED off sm_100. */
SPGEMM_API spgemm_status_t spgemm_create(spgemm_handle_t *h, int device, void *stream,
                              const spgemm_allocator_t *alloc);

/* Phase 1, steps (1)-(4) of PAPER.md:80 (Figure 1):
 *   (1) n_prod per row (Algorithm 2),
 *   (2) grouping of rows by n_prod (Table I, B200 table),
 *   (3) per-group hash counting of each row's distinct columns (Algorithms 3-5,
 *       PAPER.md:98-155) with the shared-memory -> global-memory overflow retry of
 *       PAPER.md:155, 181,
 *   (4) prefix sum into c_rpt, plus step (6) grouping by nnz for phase 2.
 * m, k, n: shapes of A (m x k) and B (k x n).  a_rpt: m+1, a_col: a_rpt[m]-a_rpt[0] used
 * entries (indexed by a_rpt values).  b_rpt: k+1, b_col.  c_rpt: m+1 int64, caller-
 * allocated, filled with c_rpt[0] = 0.  c_nnz (host): exact nnz(C).  nprod (host,
 * nullable): sum of intermediate products (the FLOPS numerator / 2).
 * Synchronises the handle's stream before returning. */
SPGEMM_API spgemm_status_t spgemm_symbolic(spgemm_handle_t h, int64_t m, int64_t k, int64_t n,
                                const int64_t *a_rpt, const int32_t *a_col,
                                const int64_t *b_rpt, const int32_t *b_col,
                                int64_t *c_rpt, int64_t *c_nnz, int64_t *nprod);

/* Phase 2, step (7) of PAPER.md:80 and §III-C: per-group hash
 * accumulation of values, gather of the non-empty entries and sort by column, written to
 * c_col / c_val (exactly c_nnz elements each, caller-allocated).  a_val / b_val: values of
 * the A and B given to the last spgemm_symbolic, both of dtype `dt`; accumulation is in
 * that working precision.  Asynchronous on the handle's stream; may be
 * called repeatedly after one symbolic (new values, same structure). */
SPGEMM_API spgemm_status_t spgemm_numeric(spgemm_handle_t h, spgemm_dtype_t dt,
                               const void *a_val, const void *b_val,
                               int32_t *c_col, void *c_val);

/* Release the handle and all library workspace. */
SPGEMM_API spgemm_status_t spgemm_destroy(spgemm_handle_t h);

SPGEMM_API const char *spgemm_status_string(spgemm_status_t s);
SPGEMM_API const char *spgemm_last_error(spgemm_handle_t h); /* owned by h; valid until next call */

/* ---------------------------------------------------------------- tuning / inspection */

typedef enum {
    SPGEMM_OPT_SYM_MIN_GROUP = 0,   /* force every row into group >= v (-1 = off); the
                                       last group index = global-memory fallback */
    SPGEMM_OPT_NUM_MIN_GROUP = 1,   /* same for the numeric grouping */
    SPGEMM_OPT_SYM_FILL_LIMIT = 2,  /* optimistic shared-memory table: abort a row after v
                                       distinct keys (default 3/4 of the table) */
    SPGEMM_OPT_STREAMS = 3,         /* 1 = one stream per group, 0 = serial */
    SPGEMM_OPT_VALIDATE = 4,        /* 1 = O(nnz) input validation in spgemm_symbolic */
    SPGEMM_OPT_LANES = 5,           /* lanes per B row (power of two 1..32), 0 = auto */
    SPGEMM_OPT_WORKSPACE_BUDGET = 6,/* max bytes for global-memory hash tables */
    SPGEMM_OPT_TIMING = 7,          /* 0 off; 1 (default) phase events, plus per-group kernel events
                                       when graphs are off; 2 per-group kernel events always (disables
                                       graph capture: events inside a graph cannot be timed) */
    SPGEMM_OPT_LONG_ROW = 8,        /* CTA-per-row groups: B rows longer than v are walked by
                                       the whole CTA (0 = auto, -1 = off) */
    SPGEMM_OPT_RANGE_HASH = 9,      /* 1 (default): rows whose column span fits the group's table
                                       use the offset hash key - lo_i (collision-free, ordered);
                                       0: the paper's multiplicative hash (Alg. 5) everywhere */
    SPGEMM_OPT_CLUSTER = 10,        /* 1 (default): rows beyond one SM's shared memory use a
                                       cluster-per-row table in distributed shared memory before
                                       the global-memory fallback; 0: straight to global memory */
    SPGEMM_OPT_CLUSTER_FILL_LIMIT = 11, /* symbolic cluster table: rows with more distinct keys
                                       than v go to global memory (0 = capacity/2) */
    SPGEMM_OPT_FLAT = 12,           /* product loop: 1 load-balanced flattened (lanes share a batch
                                       of A non-zeros), 0 VW lanes per A non-zero, -1 auto (1 when
                                       the mean B row is shorter than 16) */
    SPGEMM_OPT_GRAPHS = 13,         /* 1 (default): the asynchronous segments (phase-1 group kernels
                                       + scan, phase-2 group kernels, on their forked streams) are
                                       captured into CUDA graphs and replayed while inputs,
                                       workspace and group histogram are unchanged */
    SPGEMM_OPT_RANGE_WARP = 14,     /* 1 (default): "range rows" — exact column span R_i <= 2048,
                                       R_i <= 4 n_prod_i, n_prod_i in [RANGE_MIN_NPROD, 65536] — are
                                       counted and computed by warp-per-row kernels over an offset
                                       table of R_i slots; the count is a union of
                                       B-row bitmaps when every range row has R_i <= 1024 (and the
                                       bitmaps fit half the workspace budget), else one flag store
                                       per product.  2: range rows, flag stores always (ablation).
                                       0: Table-I groups only.  Needs RANGE_HASH; off while a
                                       MIN_GROUP is forced */
    SPGEMM_OPT_RANGE_MIN_NPROD = 15,/* n_prod lower bound of range rows (default 256) */
    SPGEMM_OPT_BITMAP_RANK = 16,    /* CTA-per-row numeric hash groups order each row by a
                                       two-level bitmap rank over its column span:
                                       1 (default) where the level-1 width n/1024 + 1 is at most
                                       the group's nnz bound, else bucket sort; 2: always;
                                       0: bucket sort everywhere (ablation) */
    SPGEMM_OPT_RANK_ACC = 17,       /* 1 (default): CTA-per-row numeric groups (4-9) accumulate each
                                       row directly at the rank of its column — the two-level
                                       bitmap over the row's span built first, used as a
                                       collision-free order-preserving hash;
                                       needs RANGE_HASH (column spans).  0: paper hash table +
                                       gather + rank; off while NUM_MIN_GROUP
                                       is forced */
    SPGEMM_OPT_TINY = 18,           /* 1 (default): numeric groups 0-1 run thread-per-row kernels
                                       with the row's table in registers, kept in column order
                                       (DESIGN.md §5.10); 2: symbolic groups 0-1 too (measured
                                       slower than the partial-warp hash there); 0: the paper's
                                       partial-warp hash groups.  Off while a MIN_GROUP is forced */
    SPGEMM_OPT_RANK_L1_PCT = 19,    /* numeric rank kernels (RANK_ACC) only for groups whose nnz
                                       bound B satisfies 100 * W <= v * B, W = level-1 bitmap
                                       words of the column range (n / 1024 + 1): wide matrices
                                       keep the paper hash on their small-row groups (the level-1
                                       clear + prefix costs more than the row).  Default 500,
                                       0 = no limit */
    SPGEMM_OPT_RANK_L1_PCT_SYM = 20,/* same for the symbolic rank-count kernels, B = the group's
                                       n_prod bound.  Default 100, 0 = no limit */
    SPGEMM_OPT_BATCH = 21,          /* batched graph-row kernels, bit mask:
                                       1 = symbolic groups 2-9 by the paper hash (Alg. 5), R rows
                                       of one group per CTA with their products flattened;
                                       2 = numeric expand-bucket-rank (ESC) for rows of symbolic
                                       groups 2-8 with 100 * n_prod_i <= ESC_PCT * nnz_i (needs
                                       RANGE_HASH: column spans).  Default 2 (the batched symbolic
                                       kernels measured slower than the per-group ones on R-MAT
                                       s22); 0 = off (ablation).
                                       Off while the matching MIN_GROUP is forced */
    SPGEMM_OPT_ESC_PCT = 22,        /* compression bound of the ESC rows (default 200: n_prod_i <=
                                       2 nnz_i) */
    SPGEMM_OPT_ESC_GROUPS = 23,     /* bit g: rows of symbolic group g (2..7) may take the ESC kernels;
                                       -1 (default) = the library's rule */
    SPGEMM_OPT_WSORT = 25,          /* warp-per-row register sort, bit mask: 1 =
                                       symbolic groups 2-5 (n_prod_i <= 1024) count distinct columns of
                                       a bitonic-sorted register row; 2 = numeric rows of those groups
                                       with 100 * n_prod_i <= ESC_PCT * nnz_i.  Default 0 (measured
                                       slower than the hash / ESC kernels: ablation) */
    SPGEMM_OPT_RANK_BIG_SYM = 26,   /* 1 (default): symbolic rows above the last n_prod bound (the
                                       optimistic group) are counted exactly by one 1024-thread CTA
                                       per row with the two-level bitmap of RANK_ACC, level 2 in
                                       chunks of 32768 blocks, when the group has
                                       at least 4 rows per SM; 2: whatever its size.  Needs
                                       RANK_ACC and the column spans.  0: the paper's chain — optimistic shared
                                       table, overflow rows recounted in cluster / global tables
                                        */
    SPGEMM_OPT_RANK_BIG_SHARED = 27,/* 1 (default): numeric rows of group 10 (8192 < nnz_i <= 24576)
                                       on the rank-big kernel keep the level-2 bitmap and its
                                       prefix in shared memory when they fit beside level 1
                                       (DESIGN.md §5.8); 0: in the per-CTA global slab; 2: one
                                       1024-thread CTA per row with the products in registers and
                                       the output reduced into C (measured equal at R-MAT s22) */
    SPGEMM_OPT_RANK_MID = 28,       /* numeric group 9 (4096 < nnz_i <= 8192) of the rank kernels
                                       (DESIGN.md §5.8): 2 (default) products held in registers,
                                       values reduced straight into the zeroed row of C at their
                                       rank, 512-thread CTAs, two per SM; 1: persistent 512-thread
                                       CTAs re-walking the products, level 2 in shared memory;
                                       0: one 1024-thread CTA per row, the row kept in shared memory */
    SPGEMM_OPT_RANK_GOUT = 29,      /* 1: numeric rank groups 3-8 reduce values straight into the
                                       zeroed row of C at their rank instead of a shared-memory
                                       row (less shared memory per CTA).  Default 0 */
    SPGEMM_OPT_RANK_BIG_MAX = 31,   /* numeric rows above the CTA groups (groups 10, 11, 12: up to
                                       24576 / 49152 / 98304 entries): the first v groups take the
                                       one-CTA-per-row rank-big kernel, the others the DSMEM cluster
                                       tables of 2/4/8 CTAs.  Default 3 */
    SPGEMM_OPT_SMALL = 24           /* 1 (default): matrices of <= 65536 rows whose rows all have
                                       n_prod_i <= 32 run each phase as one thread-per-row launch
                                       (register tables, no grouping, one host sync); otherwise,
                                       or with 0, the grouped path.  spgemm_get_grouping then
                                       returns SPGEMM_ERR_BAD_STATE */
} spgemm_option_t;

SPGEMM_API spgemm_status_t spgemm_set_option(spgemm_handle_t h, spgemm_option_t opt, int64_t value);

#define SPGEMM_MAX_GROUPS 24

/* Counters of the last symbolic/numeric call.  Times are CUDA-event milliseconds measured on
 * the stream each kernel was launched on (group kernels: their own stream). */
typedef struct {
    int64_t m, k, n, nnz_a, nnz_b, nnz_c, nprod;
    int64_t max_row_nprod, max_row_nnz;
    int32_t n_sym_groups, n_num_groups;
    int64_t sym_rows[SPGEMM_MAX_GROUPS], num_rows[SPGEMM_MAX_GROUPS];
    int64_t sym_nprod[SPGEMM_MAX_GROUPS], num_nprod[SPGEMM_MAX_GROUPS];
    int64_t sym_nnza[SPGEMM_MAX_GROUPS], num_nnza[SPGEMM_MAX_GROUPS];
    int64_t num_nnzc[SPGEMM_MAX_GROUPS];
    int64_t sym_overflow_rows;          /* rows that overflowed the one-CTA optimistic table */
    float sym_group_ms[SPGEMM_MAX_GROUPS], num_group_ms[SPGEMM_MAX_GROUPS];
    float setup_ms, symbolic_ms, scan_ms, numeric_ms; /* phases (Figure 5/6 breakdown) */
    int64_t kernel_launches_symbolic, kernel_launches_numeric;
    int64_t workspace_bytes, workspace_peak_bytes;
    int64_t sym_overflow2_rows;         /* rows that overflowed the cluster table (global memory) */
    int64_t graph_replays;              /* captured segments replayed during the last call pair */
    int32_t sym_kernel[SPGEMM_MAX_GROUPS];  /* kernel family that ran each group of the last call: */
    int32_t num_kernel[SPGEMM_MAX_GROUPS];  /* spgemm_kernel_t below (0: group empty / not run)    */
} spgemm_stats_t;

/* Kernel families reported per group in spgemm_stats_t. */
typedef enum {
    SPGEMM_KERNEL_NONE = 0,
    SPGEMM_KERNEL_HASH = 1,     /* paper hash table in shared memory (Alg. 5, Table I groups)    */
    SPGEMM_KERNEL_RANK = 2,     /* rank-indexed table, one CTA per row (kernels_rankacc.cu)      */
    SPGEMM_KERNEL_RANGE = 3,    /* range rows: offset table, warp per row (kernels_range.cu)     */
    SPGEMM_KERNEL_CLUSTER = 4,  /* distributed shared-memory hash table (kernels_cluster.cu)     */
    SPGEMM_KERNEL_GLOBAL = 5,   /* global-memory hash table                  */
    SPGEMM_KERNEL_RANK_BIG = 6, /* rank-indexed, level 2 in global memory, values reduced into C */
    SPGEMM_KERNEL_TINY = 7,     /* thread per row, sorted register table (kernels_tiny.cu)       */
    SPGEMM_KERNEL_BATCH = 8,    /* batched rows per CTA, paper hash in shared memory (symbolic)   */
    SPGEMM_KERNEL_ESC = 9,      /* batched expand-bucket-rank-compress rows (kernels_esc.cu)      */
    SPGEMM_KERNEL_WSORT = 10    /* warp per row, bitonic-sorted register row (kernels_wsort.cu)   */
} spgemm_kernel_t;

SPGEMM_API spgemm_status_t spgemm_get_stats(spgemm_handle_t h, spgemm_stats_t *out /* host */);

/* Group table of the implementation: inclusive upper bounds of each group's key (n_prod
 * for phase 1, nnz for phase 2), ascending; the group after the last bound is the global-
 * memory fallback.  *ngroups (host) receives the number of bounds. */
SPGEMM_API spgemm_status_t spgemm_group_bounds(int phase /* 1 or 2 */, int64_t *upper /* host, >= 24 */,
                                    int32_t *ngroups /* host */);

/* Copy the per-row n_prod (int64, m) and the grouping permutation of `phase` (int32, m:
 * row ids concatenated group by group) plus group offsets (int64, ngroups+2) of the last
 * symbolic call to HOST buffers (for tests). */
SPGEMM_API spgemm_status_t spgemm_get_grouping(spgemm_handle_t h, int phase, int64_t *nprod,
                                    int32_t *perm, int64_t *offsets);

/* Multi-GPU row partition: n_prod-balanced contiguous row blocks of A for nparts ranks.
 * splits (host, nparts+1): splits[0] = 0, splits[nparts] = m, and block p holds rows
 * [splits[p], splits[p+1]) with prefix(n_prod) crossing p*total/nparts at its start. */
SPGEMM_API spgemm_status_t spgemm_row_partition(spgemm_handle_t h, int64_t m, int64_t k,
                                     const int64_t *a_rpt, const int32_t *a_col,
                                     const int64_t *b_rpt, int32_t nparts, int64_t *splits);

/* Library build info, e.g. "spgemm sm_100a <date>" (static string). */
SPGEMM_API const char *spgemm_version(void);

#ifdef __cplusplus
}
#endif
#endif /* SPGEMM_H_ */
