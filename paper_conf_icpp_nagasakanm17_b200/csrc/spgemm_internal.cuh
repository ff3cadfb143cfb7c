// spgemm_internal.cuh — group tables, device primitives and launcher declarations shared by
// the kernels of libspgemm.so (B200 / sm_100a).  Nothing here is shared with oracle/.
//
// Paper map (PAPER.md line numbers):
//   Alg. 2 n_prod count ........ :90-96   -> k_nprod_group       (kernels_setup.cu)
//   grouping (2)/(6) ........... :84-88   -> k_group_scatter     (kernels_setup.cu)
//   Alg. 3/4 thread assignment . :102-126 -> sym_row / num_row   (sub-groups of VW lanes)
//   Alg. 5 hash insert ......... :130-153 -> hash_insert / hash_slot (below)
//   group-0 overflow retry ..... :155,181 -> optimistic group + k_sym_global
//   calculation + gather + sort  :171-173 -> num_row (bucket-rank sort)
//   Table I / parameter rule ... :157-183 -> kSymGroups / kNumGroups (B200 values)
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

namespace spg {

constexpr unsigned kHashScal = 107u;  // HASH_SCAL; any odd constant (reading R4)
constexpr int kMaxGroups = 16;
constexpr int kSmemLimit = 232448;     // 227 KB opt-in per CTA on sm_100

// ----------------------------------------------------------------------------- group tables
// B200 re-derivation of Table I: power-of-two tables,
// table >= 2x the group's key bound (load factor <= 1/2 for linear probing), threads per row
// (TPR) ~ key bound / 4..8, one row per CTA once TPR > 32 (TB/ROW), several rows per CTA
// below (PWARP/ROW generalised to 4/8/16/32 lanes).
struct GroupSpec {
  long long upper;  // inclusive upper bound of the group key (n_prod or nnz)
  int T;            // hash table slots
  int TPR;          // threads per row
  int BS;           // threads per CTA
};

// Phase 1 (symbolic), key = n_prod_i.  Group 10 is the OPTIMISTIC shared-memory attempt for
// rows above the last bound ("using the maximum hash table size for shared
// memory"); rows that find more than the fill limit of distinct keys are retried in global
// memory (group kSymGlobal).
constexpr GroupSpec kSymGroups[] = {
    {16, 32, 4, 256},        {32, 64, 8, 256},         {128, 256, 16, 256},
    {256, 512, 32, 256},     {512, 1024, 64, 64},      {1024, 2048, 128, 128},
    {2048, 4096, 256, 256},  {4096, 8192, 512, 512},   {8192, 16384, 1024, 1024},
    {16384, 32768, 1024, 1024},
    {-1, 32768, 1024, 1024},  // optimistic (no upper bound)
};
constexpr int kNumSymBounds = 10;   // groups 0..9 have an upper bound
constexpr int kSymOptimistic = 10;
constexpr int kSymGlobal = 11;
constexpr int kNumSymGroups = 12;   // including global

// Phase 2 (numeric), key = nnz_i.  Same bounds for fp32 and fp64 (fp64 sizes the smem).
constexpr GroupSpec kNumGroups[] = {
    {8, 16, 4, 256},         {16, 32, 8, 256},         {64, 128, 16, 256},
    {128, 256, 32, 256},     {256, 512, 64, 64},       {512, 1024, 128, 128},
    {1024, 2048, 256, 256},  {2048, 4096, 512, 512},   {4096, 8192, 1024, 1024},
    {8192, 16384, 1024, 1024},
};
constexpr int kNumNumBounds = 10;
constexpr int kNumGlobal = 10;
constexpr int kNumNumGroups = 11;

// Numeric per-row shared-memory layout: vals[T] | keys[T] | bucket[NB+1] | sidx[upper] ,
// NB = T/4 buckets for the bucket-rank sort.
__host__ __device__ constexpr int num_nbuckets(int T) { return T / 4; }
__host__ __device__ constexpr int align16(int x) { return (x + 15) & ~15; }
template <typename VT>
__host__ __device__ constexpr int num_row_bytes(int T, long long upper) {
  return align16(T * (int)sizeof(VT) + T * 4 + (num_nbuckets(T) + 1) * 4 + (int)upper * 2 + 8);
}

// ----------------------------------------------------------------------------- device state
struct DevAcc {  // zeroed at the start of spgemm_symbolic, copied to pinned host at the syncs
  unsigned long long total_nprod;
  unsigned long long max_nprod;
  unsigned long long max_nnz;
  unsigned long long sym_rows[kMaxGroups], sym_nprod[kMaxGroups], sym_nnza[kMaxGroups];
  unsigned long long num_rows[kMaxGroups], num_nprod[kMaxGroups], num_nnza[kMaxGroups];
  unsigned long long num_nnzc[kMaxGroups];
  long long nnzc;
  int overflow_count;
  int err_flags;  // bit0 invalid input, bit1 numeric row count mismatch
  int cursor[2][kMaxGroups];
};

struct Bounds {  // group bounds passed by value
  long long upper[kMaxGroups];
  int nbounds;     // groups 0..nbounds-1 bounded; key > last bound -> group nbounds
  int min_group;   // -1 or forced minimum group
};

struct Offsets {
  long long off[kMaxGroups + 1];
  int ngroups;
};

// ----------------------------------------------------------------------------- primitives
__device__ __forceinline__ int ld_volatile(const int* p) { return *(const volatile int*)p; }

// Algorithm 5: key = col_B[k]; hash = key*HASH_SCAL mod t_size (t_size a
// power of two -> mask); linear probing; empty = -1; insert by atomicCAS.
// Returns 1 if this call inserted the key (nz <- nz + 1), else 0.
__device__ __forceinline__ int hash_insert(int* table, unsigned mask, int key) {
  unsigned h = ((unsigned)key * kHashScal) & mask;
  while (true) {
    int cur = ld_volatile(table + h);
    if (cur == key) return 0;
    if (cur == -1) {
      int old = atomicCAS(table + h, -1, key);
      if (old == -1) return 1;
      if (old == key) return 0;
    }
    h = (h + 1) & mask;
  }
}

// Same probe, returning the slot (numeric phase, "utilizing hash table as well").
__device__ __forceinline__ unsigned hash_slot(int* table, unsigned mask, int key, bool& inserted) {
  unsigned h = ((unsigned)key * kHashScal) & mask;
  while (true) {
    int cur = ld_volatile(table + h);
    if (cur == key) { inserted = false; return h; }
    if (cur == -1) {
      int old = atomicCAS(table + h, -1, key);
      if (old == -1) { inserted = true; return h; }
      if (old == key) { inserted = false; return h; }
    }
    h = (h + 1) & mask;
  }
}

// Row-group collectives: TPR <= 32 -> lanes of one warp (shuffles with width TPR);
// TPR > 32 -> the whole CTA (one row per CTA), ws = >= 33 ints of shared scratch.
template <int TPR>
struct Grp {
  static __device__ __forceinline__ void sync() {
    if constexpr (TPR <= 32) __syncwarp(); else __syncthreads();
  }
  static __device__ __forceinline__ int lane() { return threadIdx.x % TPR; }

  // exclusive prefix of v over the group; *total receives the group sum.
  static __device__ __forceinline__ long long excl_scan(long long v, long long* total, long long* ws) {
    if constexpr (TPR <= 32) {
      long long x = v;
#pragma unroll
      for (int d = 1; d < TPR; d <<= 1) {
        long long y = __shfl_up_sync(0xffffffffu, x, d, TPR);
        if (lane() >= d) x += y;
      }
      *total = __shfl_sync(0xffffffffu, x, TPR - 1, TPR);
      return x - v;
    } else {
      constexpr int NW = TPR / 32;
      const int l = threadIdx.x & 31, w = threadIdx.x >> 5;
      long long x = v;
#pragma unroll
      for (int d = 1; d < 32; d <<= 1) {
        long long y = __shfl_up_sync(0xffffffffu, x, d);
        if (l >= d) x += y;
      }
      __syncthreads();  // protect ws from a previous use
      if (l == 31) ws[w] = x;
      __syncthreads();
      if (w == 0) {
        long long s = (l < NW) ? ws[l] : 0;
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) {
          long long y = __shfl_up_sync(0xffffffffu, s, d);
          if (l >= d) s += y;
        }
        if (l < NW) ws[l] = s;  // inclusive warp totals
      }
      __syncthreads();
      long long base = (w > 0) ? ws[w - 1] : 0;
      *total = ws[NW - 1];
      return base + x - v;
    }
  }

  static __device__ __forceinline__ long long sum(long long v, long long* ws) {
    long long t;
    excl_scan(v, &t, ws);
    return t;
  }
};

// ----------------------------------------------------------------------------- launchers
struct SymArgs {
  const int64_t* a_rpt; const int32_t* a_col;
  const int64_t* b_rpt; const int32_t* b_col;
  const int32_t* rows;     // permutation segment of this group
  long long nrows;
  int64_t* c_cnt;          // c_rpt + 1: per-row nnz written here (scanned later)
  int vw_log2;             // lanes per B row = 1 << vw_log2 (Alg. 3/4 generalised)
  // optimistic group
  int32_t* overflow_rows; int* overflow_count; int fill_limit;
  // global fallback
  int* slab; long long slab_T; const int64_t* nprod; long long n;
  const int* dev_count;    // extra rows from overflow list (device count), may be null
};

struct NumArgs {
  const int64_t* a_rpt; const int32_t* a_col; const void* a_val;
  const int64_t* b_rpt; const int32_t* b_col; const void* b_val;
  const int32_t* rows; long long nrows;
  const int64_t* c_rpt; int32_t* c_col; void* c_val;
  int vw_log2;
  int* err_flags;
  // global fallback
  void* slab; long long slab_T; long long slab_stride; long long max_nnz;
};

cudaError_t launch_nprod_group(cudaStream_t s, long long m, const int64_t* a_rpt, const int32_t* a_col,
                               const int64_t* b_rpt, int64_t* nprod, uint8_t* grp, int64_t* c_rpt,
                               DevAcc* acc, Bounds b, int lpr_log2);
cudaError_t launch_group_scatter(cudaStream_t s, long long m, const uint8_t* grp, Offsets off,
                                 int* cursor, int32_t* perm);
cudaError_t launch_scan_and_group(cudaStream_t s, long long m, int64_t* c_rpt, const int64_t* nprod,
                                  const int64_t* a_rpt, uint8_t* grp2, DevAcc* acc, Bounds b,
                                  long long* tile_ws, int* nlaunch);
size_t scan_workspace_bytes(long long m);
cudaError_t launch_validate(cudaStream_t s, long long m, long long k, long long n, const int64_t* a_rpt,
                            const int32_t* a_col, const int64_t* b_rpt, const int32_t* b_col, int* err);
cudaError_t launch_partition(cudaStream_t s, long long m, const int64_t* a_rpt, const int32_t* a_col,
                             const int64_t* b_rpt, int64_t* nprod_scan, long long* tile_ws,
                             int nparts, int64_t* splits_dev, int* nlaunch);

cudaError_t launch_symbolic_group(cudaStream_t s, int group, const SymArgs& a, int num_sms);
cudaError_t launch_symbolic_global(cudaStream_t s, const SymArgs& a, int grid);
cudaError_t launch_numeric_group(cudaStream_t s, int group, bool fp64, const NumArgs& a);
cudaError_t launch_numeric_global(cudaStream_t s, bool fp64, const NumArgs& a, int grid);

}  // namespace spg
