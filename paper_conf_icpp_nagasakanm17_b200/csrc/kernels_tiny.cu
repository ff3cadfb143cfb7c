// kernels_tiny.cu — thread-per-row kernels for the smallest groups (B200 addition, DESIGN.md
// §5.10): symbolic groups 0-1 (n_prod_i <= 32) and numeric groups 0-1 (nnz_i <= 16).
//
// The paper gives its smallest rows a "partial warp" (PWARP/ROW) and a small
// shared-memory hash table per row.  For rows of a handful of products (web graphs: 83 % of the
// webbase-like rows have nnz_i <= 8; the Epidemiology-like torus has 16 products and 10 outputs per
// row) the table initialisation, the probing and the per-row sort of the table cost more than the
// products.  Here one thread owns a row and keeps its table in registers, in column order:
//
//   * the row's products are walked in Alg. 1 order: A non-zeros j in order, B
//     entries q in order;
//   * each product is inserted into a sorted register array of at most CAP distinct columns
//     (CAP >= nnz_i for numeric rows: the symbolic count of the group bound; >= n_prod_i for
//     symbolic rows): a compare pass counts the smaller keys and detects an equal one (the
//     table lookup of Alg. 5), an equal key accumulates (numeric: value += a_ik * b_kj, in the
//     working precision), a new key is inserted at its rank (shifting the larger
//     ones) — "insert if absent, else accumulate" (reading R1), with the sort of PAPER.md:173
//     maintained on the fly;
//   * symbolic: nnz_i = number of distinct keys; numeric: the array is row i of C.
//
// Register arrays are indexed only with compile-time indices (fully unrolled, predicated), so
// nothing spills to local memory.  Values are summed in the order Alg. 1 visits the products
// (deterministic).
#include <climits>

#include "spgemm_internal.cuh"

namespace spg {

namespace {

// Sorted insertion of (key, x) into k[0..n) / v[0..n) (CAP registers each).
template <typename VT, int CAP, bool NUM>
__device__ __forceinline__ void tiny_insert(int (&k)[CAP], VT (&v)[CAP], int& n, int key, VT x, bool& overflow) {
  int below = 0;
  bool eq = false;
#pragma unroll
  for (int s = 0; s < CAP; ++s) {
    const bool live = s < n;
    below += live && k[s] < key;
    eq |= live && k[s] == key;
  }
  if (eq) {
    if constexpr (NUM) {
#pragma unroll
      for (int s = 0; s < CAP; ++s)
        if (s == below) v[s] += x;
    }
    return;
  }
  if (n >= CAP) {  // more distinct keys than the group allows: inconsistent input
    overflow = true;
    return;
  }
#pragma unroll
  for (int s = CAP - 1; s > 0; --s)
    if (s > below) {
      k[s] = k[s - 1];
      if constexpr (NUM) v[s] = v[s - 1];
    }
#pragma unroll
  for (int s = 0; s < CAP; ++s)
    if (s == below) {
      k[s] = key;
      if constexpr (NUM) v[s] = x;
    }
  ++n;
}

// Walk the products of `row` in Alg. 1 order, calling f(key, a_ik * b_kj).
template <bool NUM, typename VT, typename F>
__device__ __forceinline__ void tiny_products(const int64_t* __restrict__ a_rpt, const int32_t* __restrict__ a_col,
                                              const VT* __restrict__ a_val, const int64_t* __restrict__ b_rpt,
                                              const int32_t* __restrict__ b_col, const VT* __restrict__ b_val,
                                              int row, F&& f) {
  const long long a0 = __ldg(a_rpt + row), a1 = __ldg(a_rpt + row + 1);
  for (long long j = a0; j < a1; ++j) {
    const int kk = __ldg(a_col + j);
    const VT av = NUM ? __ldg(a_val + j) : VT(0);
    const long long q0 = __ldg(b_rpt + kk), q1 = __ldg(b_rpt + kk + 1);
    long long q = q0;
    // two B entries per step: both loads in flight before the inserts
    for (; q + 1 < q1; q += 2) {
      const int k0 = __ldg(b_col + q), k1 = __ldg(b_col + q + 1);
      const VT w0 = NUM ? __ldg(b_val + q) : VT(0), w1 = NUM ? __ldg(b_val + q + 1) : VT(0);
      f(k0, av * w0);
      f(k1, av * w1);
    }
    if (q < q1) f(__ldg(b_col + q), NUM ? av * __ldg(b_val + q) : VT(0));
  }
}

template <int CAP>
__global__ __launch_bounds__(128) void k_sym_tiny(SymArgs a) {
  const long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= a.nrows) return;
  const int row = a.rows[i];
  int k[CAP];
  int dummy[CAP];
  int n = 0;
  bool overflow = false;
#pragma unroll
  for (int s = 0; s < CAP; ++s) k[s] = INT_MAX;
  tiny_products<false, int>(a.a_rpt, a.a_col, nullptr, a.b_rpt, a.b_col, nullptr, row,
                            [&](int key, int) { tiny_insert<int, CAP, false>(k, dummy, n, key, 0, overflow); });
  a.c_cnt[row] = n;
  if (overflow) atomicOr(a.err_flags, 1);
}

template <typename VT, int CAP>
__global__ __launch_bounds__(128) void k_num_tiny(NumArgs a) {
  const long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= a.nrows) return;
  const int row = a.rows[i];
  int k[CAP];
  VT v[CAP];
  int n = 0;
  bool overflow = false;
#pragma unroll
  for (int s = 0; s < CAP; ++s) { k[s] = INT_MAX; v[s] = VT(0); }
  tiny_products<true, VT>(a.a_rpt, a.a_col, static_cast<const VT*>(a.a_val), a.b_rpt, a.b_col,
                          static_cast<const VT*>(a.b_val), row,
                          [&](int key, VT x) { tiny_insert<VT, CAP, true>(k, v, n, key, x, overflow); });
  const long long c0 = a.c_rpt[row];
  const int cn = (int)(a.c_rpt[row + 1] - c0);
  if (overflow || n != cn) atomicOr(a.err_flags, 2);
  int32_t* __restrict__ cc = a.c_col + c0;
  VT* __restrict__ cv = static_cast<VT*>(a.c_val) + c0;
#pragma unroll
  for (int s = 0; s < CAP; ++s)
    if (s < n && s < cn) {
      cc[s] = k[s];
      cv[s] = v[s];
    }
}

// Small matrices (m <= kSmallRows), whole phases in one launch each, a WARP per row and a lane
// per product (rows with nnz(A_i) <= 32 and n_prod_i <= 32; a row above flags an overflow and the
// host runs the general grouped path instead).  n_prod_i (Alg. 2) comes from the same pass.  The
// row's loads take four dependent rounds whatever its shape (a_rpt; col_A, one per lane; the
// rpt_B pairs; one B entry per lane), the products are ordered by a 32-lane bitonic network on
// (column, value) pairs, equal columns are adjacent and summed (numeric, working precision,
// PAPER.md:179), and each distinct column's position is the count of distinct columns below it
// (PAPER.md:173's rank): no grouping, no shared memory, no sync 1.
constexpr unsigned kFullW = 0xffffffffu;

template <bool NUM, typename VT>
__device__ __forceinline__ bool small_warp_row(const int64_t* __restrict__ a_rpt, const int32_t* __restrict__ a_col,
                                               const VT* __restrict__ a_val, const int64_t* __restrict__ b_rpt,
                                               const int32_t* __restrict__ b_col, const VT* __restrict__ b_val,
                                               int row, int lane, int& key, VT& val, long long& np_out) {
  const long long a0 = __ldg(a_rpt + row), a1 = __ldg(a_rpt + row + 1);
  const int na = (int)(a1 - a0);
  np_out = 33;
  if (na > 32) return false;  // warp-uniform: the grouped path takes this matrix
  long long b0 = 0;
  int len = 0;
  VT av = VT(0);
  if (lane < na) {
    const int kk = __ldg(a_col + a0 + lane);
    if (NUM) av = __ldg(a_val + a0 + lane);
    b0 = __ldg(b_rpt + kk);
    len = (int)(__ldg(b_rpt + kk + 1) - b0);
  }
  long long np = len;
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) np += __shfl_xor_sync(kFullW, np, o);
  np_out = np;
  if (np > 32) return false;  // warp-uniform
  int incl = len;
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    const int y = __shfl_up_sync(kFullW, incl, d);
    if (lane >= d) incl += y;
  }
  // product `lane` (Alg. 1 order) -> entry e = #entries whose inclusive prefix <= lane
  int ent = 0;
#pragma unroll
  for (int st = 16; st > 0; st >>= 1)
    if (__shfl_sync(kFullW, incl, ent + st - 1) <= lane) ent += st;
  const int ex = __shfl_sync(kFullW, incl - len, ent);
  const long long eb = __shfl_sync(kFullW, b0, ent);
  const VT ea = NUM ? __shfl_sync(kFullW, av, ent) : VT(0);
  key = INT_MAX;
  val = VT(0);
  if (lane < np) {
    const long long q = eb + (lane - ex);
    key = __ldg(b_col + q);
    if (NUM) val = ea * __ldg(b_val + q);
  }
  // bitonic sort of (key, val) over the 32 lanes, ascending
#pragma unroll
  for (int k = 2; k <= 32; k <<= 1) {
#pragma unroll
    for (int j = k >> 1; j > 0; j >>= 1) {
      const int ok = __shfl_xor_sync(kFullW, key, j);
      const VT ov = NUM ? __shfl_xor_sync(kFullW, val, j) : VT(0);
      const bool up = (lane & k) == 0;           // this pair sorts ascending
      const bool lower = (lane & j) == 0;        // this lane keeps the smaller key
      const bool take = up == lower ? ok < key : ok > key;
      if (take) {
        key = ok;
        if (NUM) val = ov;
      }
    }
  }
  return true;
}

__global__ __launch_bounds__(128) void k_small_sym(long long m, long long k, const int64_t* __restrict__ a_rpt,
                                                   const int32_t* __restrict__ a_col, const int64_t* __restrict__ b_rpt,
                                                   const int32_t* __restrict__ b_col, int64_t* __restrict__ c_cnt,
                                                   int64_t* __restrict__ nprod, DevAcc* acc) {
  const long long row = ((long long)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int lane = threadIdx.x & 31;
  if (row == 0 && lane == 0) {  // what the host needs besides nnz(C): nnz(A), nnz(B)
    acc->ends[0] = a_rpt[0]; acc->ends[1] = a_rpt[m]; acc->ends[2] = b_rpt[0]; acc->ends[3] = b_rpt[k];
  }
  if (row >= m) return;  // warp-uniform
  int key;
  int dummy;
  long long np;
  const bool fast = small_warp_row<false, int>(a_rpt, a_col, nullptr, b_rpt, b_col, nullptr, (int)row, lane, key,
                                               dummy, np);
  int n = 0;
  if (fast) {
    const int prev = __shfl_up_sync(kFullW, key, 1);
    n = __popc(__ballot_sync(kFullW, key != INT_MAX && (lane == 0 || prev != key)));
  } else if (np > 0 && lane == 0) {
    atomicAdd(&acc->small_overflow, 1);
  }
  if (lane == 0) {
    nprod[row] = np;
    c_cnt[row] = n;
    atomicAdd(&acc->total_nprod, (unsigned long long)np);
    atomicMax(&acc->max_nprod, (unsigned long long)np);
  }
}

template <typename VT>
__global__ __launch_bounds__(128) void k_small_num(NumArgs a, long long m) {
  const long long row = ((long long)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int lane = threadIdx.x & 31;
  if (row >= m) return;  // warp-uniform
  int key;
  VT val;
  long long np;
  const bool fast = small_warp_row<true, VT>(a.a_rpt, a.a_col, static_cast<const VT*>(a.a_val), a.b_rpt, a.b_col,
                                             static_cast<const VT*>(a.b_val), (int)row, lane, key, val, np);
  const long long c0 = a.c_rpt[row];
  const int cn = (int)(a.c_rpt[row + 1] - c0);
  if (!fast) {
    if (np > 0 && lane == 0) atomicOr(a.err_flags, 2);
    return;
  }
  const int prev = __shfl_up_sync(kFullW, key, 1);
  const bool head = key != INT_MAX && (lane == 0 || prev != key);
  // sum each run of equal keys into its head: segmented suffix sums over the lanes
  VT run = val;
  int seg = key;
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    const VT y = __shfl_down_sync(kFullW, run, d);
    const int ky = __shfl_down_sync(kFullW, seg, d);
    if (lane + d < 32 && ky == key) run += y;
  }
  const unsigned hm = __ballot_sync(kFullW, head);
  if (__popc(hm) != cn) {
    if (lane == 0) atomicOr(a.err_flags, 2);
    return;
  }
  if (head) {
    const int pos = __popc(hm & ((1u << lane) - 1u));
    a.c_col[c0 + pos] = key;
    static_cast<VT*>(a.c_val)[c0 + pos] = run;
  }
}

}  // namespace

cudaError_t launch_small_symbolic(cudaStream_t s, long long m, long long k, const int64_t* a_rpt, const int32_t* a_col,
                                  const int64_t* b_rpt, const int32_t* b_col, int64_t* c_cnt, int64_t* nprod,
                                  DevAcc* acc) {
  if (m <= 0) return cudaSuccess;
  k_small_sym<<<(unsigned)((m * 32 + 127) / 128), 128, 0, s>>>(m, k, a_rpt, a_col, b_rpt, b_col, c_cnt, nprod, acc);
  return cudaGetLastError();
}

cudaError_t launch_small_numeric(cudaStream_t s, bool fp64, const NumArgs& a, long long m) {
  if (m <= 0) return cudaSuccess;
  const unsigned grid = (unsigned)((m * 32 + 127) / 128);
  if (fp64) k_small_num<double><<<grid, 128, 0, s>>>(a, m);
  else k_small_num<float><<<grid, 128, 0, s>>>(a, m);
  return cudaGetLastError();
}

// Groups served (capacity = the group's bound): symbolic 0 (n_prod <= 16), 1 (<= 32); numeric 0
// (nnz <= 8), 1 (<= 16).
bool tiny_group(int phase, int group) {
  if (phase == 1) return group == 0 || group == 1;
  return group == 0 || group == 1;
}

cudaError_t launch_symbolic_tiny(cudaStream_t s, int group, const SymArgs& a) {
  if (a.nrows <= 0) return cudaSuccess;
  const unsigned grid = (unsigned)((a.nrows + 127) / 128);
  static_assert(kSymGroups[0].upper == 16 && kSymGroups[1].upper == 32, "tiny symbolic capacities");
  if (group == 0) k_sym_tiny<16><<<grid, 128, 0, s>>>(a);
  else if (group == 1) k_sym_tiny<32><<<grid, 128, 0, s>>>(a);
  else return cudaErrorInvalidValue;
  return cudaGetLastError();
}

cudaError_t launch_numeric_tiny(cudaStream_t s, int group, bool fp64, const NumArgs& a) {
  if (a.nrows <= 0) return cudaSuccess;
  const unsigned grid = (unsigned)((a.nrows + 127) / 128);
  static_assert(kNumGroups[0].upper == 8 && kNumGroups[1].upper == 16, "tiny numeric capacities");
  if (group == 0) {
    if (fp64) k_num_tiny<double, 8><<<grid, 128, 0, s>>>(a);
    else k_num_tiny<float, 8><<<grid, 128, 0, s>>>(a);
  } else if (group == 1) {
    if (fp64) k_num_tiny<double, 16><<<grid, 128, 0, s>>>(a);
    else k_num_tiny<float, 16><<<grid, 128, 0, s>>>(a);
  } else {
    return cudaErrorInvalidValue;
  }
  return cudaGetLastError();
}

}  // namespace spg
