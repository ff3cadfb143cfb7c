// kernels_symbolic.cu — step (3) of PAPER.md:80: count nnz of each row of C with per-row
// hash tables (§III-B), one kernel per group (Table I, B200 values in
// spgemm_internal.cuh).
//
// Thread assignment (Alg. 3/4) generalised in for_each_product: a row is
// owned by TPR threads (4..32 lanes = the PWARP/ROW family, or a whole CTA = TB/ROW); inside
// the row, sub-groups of VW lanes take successive non-zeros of A (Alg. 4 "one warp for each
// non-zero element of matrix A") and stride VW over the B row (Alg. 4 "one thread for each
// non-zero element of matrix B").  VW = 1 is exactly Alg. 3.
//
// Hash table: Alg. 5 in shared memory, t_size a power of two >= 2x the group's n_prod bound,
// so it cannot overflow.  The optimistic group (rows above the last bound) uses the largest
// table and aborts a row once it has found `fill_limit` distinct keys; the row index is
// recorded and the row is recounted in a global-memory table sized from its n_prod
// by k_sym_global.
#include <type_traits>

#include "spgemm_internal.cuh"

namespace spg {

namespace {

struct NoStop {
  __device__ __forceinline__ bool operator()() const { return false; }
};

// The product loop of one symbolic row: CTA-per-row groups in flat mode use the block-level
// flattened loop; otherwise the per-sub-group loop plus the CTA pass over deferred long B rows.
template <bool STOP, int TPR, typename BF, typename F, typename S>
__device__ __forceinline__ void sym_products(const SymArgs& a, bool active, int row, int t, int long_len,
                                             int* s_list, int& s_lcnt, BF* bf, long long* ws, F&& f,
                                             S&& stop) {
  if constexpr (TPR > 32) {
    if (a.flat) {
      for_each_product_block<false, STOP, int, TPR>(a.a_rpt, a.a_col, nullptr, a.b_rpt, a.b_col, nullptr, active, row,
                                                    t, bf, ws, f, stop);
      return;
    }
  }
  if (active)
    products<false, STOP, int, TPR>(a.flat, a.a_rpt, a.a_col, nullptr, a.b_rpt, a.b_col, nullptr, row, t, TPR,
                                    a.vw_log2, f, stop, long_len, &s_lcnt);
  if constexpr (TPR > 32) {
    if (long_len > 0)
      for_long_products<false, STOP, int>(a.a_rpt, a.a_col, nullptr, a.b_rpt, a.b_col, nullptr, active, row, t, TPR,
                                          long_len, s_list, &s_lcnt, bf, f, stop);
  }
}

// One row (all TPR threads of its row group call it; the table is the group's slice).
template <int T, int TPR, bool OPT, typename BF>
__device__ __forceinline__ void sym_row(const SymArgs& a, bool active, int row, int t, int* table, long long* ws,
                                        int& s_cnt, int& s_abort, int& s_lcnt, int* s_list, BF* bf) {
  // Range-offset hash: when the row's column span R fits 4*T bytes the table
  // is a byte-flag array indexed by key - lo_i (collision-free; idempotent plain stores, no
  // atomics, conflict-free for consecutive keys); the count is the number of set flags.
  // Spans up to 32*T columns use a bitmap instead (red.shared.or; wider spans mean fewer
  // same-word collisions inside a warp).
  bool direct = false, bitmap = false;
  int lo = 0, words = 0;
  if (active && a.rlohi != nullptr) {
    const int2 r = __ldg(a.rlohi + row);
    const long long R = (long long)r.y - r.x + 1;
    if (R > 0 && R <= 4LL * T) { direct = true; lo = r.x; words = (int)((R + 3) >> 2); }
    else if (R > 0 && R <= 32LL * T) { direct = bitmap = true; lo = r.x; words = (int)((R + 31) >> 5); }
  }
  int4* t4 = reinterpret_cast<int4*>(table);
  if (direct) {
    for (int s = t; s < (words + 3) / 4; s += TPR) t4[s] = make_int4(0, 0, 0, 0);
  } else {
#pragma unroll 4
    for (int s = t; s < T / 4; s += TPR) t4[s] = make_int4(-1, -1, -1, -1);
  }
  if (OPT && threadIdx.x == 0) { s_cnt = 0; s_abort = 0; }
  if (threadIdx.x == 0) s_lcnt = 0;
  Grp<TPR>::sync();

  int cnt = 0;
  const unsigned tb = smem_u32(table);
  const SKeys K{tb};
  const int long_len = TPR > 32 ? a.long_len : 0;
  if (direct) {  // uniform within the row group (CTA-uniform when TPR > 32)
    auto f = [&](int key, int) {
      const unsigned d = (unsigned)(key - lo);
      if (bitmap) red_or_s(tb + 4u * (d >> 5), 1u << (d & 31));
      else st_s8(tb + d, 1);
    };
    sym_products<false, TPR>(a, active, row, t, long_len, s_list, s_lcnt, bf, ws, f, NoStop{});
    Grp<TPR>::sync();
    for (int w = t; w < words; w += TPR) cnt += __popc((unsigned)table[w]);  // 0/1 bytes or bits
    const int tot = Grp<TPR>::sum32(cnt, reinterpret_cast<int*>(ws));
    if (t == 0 && row >= 0) a.c_cnt[row] = tot;
    return;
  }
  if constexpr (OPT) {
    const unsigned ab = smem_u32(&s_abort);
    auto stop = [ab]() { return lds_s32(ab) != 0; };
    auto f = [&](int key, int) {
      bool ins;
      probe(K, T - 1, key, ins);
      if (ins && atomicAdd(&s_cnt, 1) + 1 >= a.fill_limit) s_abort = 1;
    };
    sym_products<true, TPR>(a, active, row, t, long_len, s_list, s_lcnt, bf, ws, f, stop);
  } else {
    auto f = [&](int key, int) {
      bool ins;
      probe(K, T - 1, key, ins);
      cnt += ins;
    };
    sym_products<false, TPR>(a, active, row, t, long_len, s_list, s_lcnt, bf, ws, f, NoStop{});
  }
  if constexpr (OPT) {
    __syncthreads();
    if (threadIdx.x == 0 && row >= 0) {
      if (s_abort) {
        const int p = atomicAdd(a.overflow_count, 1);
        a.overflow_rows[p] = row;  // PAPER.md:155 "records the row index, and immediately terminates"
      } else {
        a.c_cnt[row] = s_cnt;
      }
    }
  } else {
    const int tot = Grp<TPR>::sum32(cnt, reinterpret_cast<int*>(ws));
    if (t == 0 && row >= 0) a.c_cnt[row] = tot;
  }
}

template <int T, int TPR, int BS, bool OPT>
__global__ __launch_bounds__(BS) void k_sym_smem(SymArgs a) {
  extern __shared__ __align__(16) int smem[];
  __shared__ long long ws[33];
  __shared__ int s_cnt, s_abort, s_lcnt;
  __shared__ int s_list[TPR > 32 ? kLongChunk : 1];
  using BF = BlockFlat<int, flat_chunk_of<TPR>(), (TPR > 32 ? 4 * flat_chunk_of<TPR>() : 0)>;
  __shared__ std::conditional_t<(TPR > 32), BF, int> s_bf_store;  // only CTA groups need it
  constexpr int RPB = BS / TPR;
  static_assert(BS % TPR == 0 && (TPR <= 32 || TPR == BS), "row group must be sub-warp or the CTA");
  const int g = threadIdx.x / TPR, t = threadIdx.x % TPR;
  int* table = smem + g * T;
  const long long ridx = (long long)blockIdx.x * RPB + g;
  const bool active = ridx < a.nrows;
  const int row = active ? a.rows[ridx] : -1;
  sym_row<T, TPR, OPT>(a, active, row, t, table, ws, s_cnt, s_abort, s_lcnt, s_list,
                       reinterpret_cast<BF*>(&s_bf_store));
}

// Global-memory table per CTA (slab of slab_T ints), one row at a time; table size
// next_pow2(2*min(n_prod_i, n)) so load factor <= 1/2 ("enough large hash table
// on global memory ... set based on the number of intermediate products").
__global__ __launch_bounds__(1024) void k_sym_global(SymArgs a) {
  __shared__ long long ws[33];
  __shared__ int s_list[kLongChunk], s_lcnt;
  __shared__ BlockFlat<int> s_bf;
  int* table = a.slab + (long long)blockIdx.x * a.slab_T;
  const long long nA = a.nrows;
  const long long nB = a.dev_count2 ? (long long)*a.dev_count2 : 0;
  const int t = threadIdx.x;
  for (long long i = blockIdx.x; i < nA + nB; i += gridDim.x) {
    const int row = i < nA ? a.rows[i] : a.overflow2_rows[i - nA];
    const long long cap = a.nprod[row] < a.n ? a.nprod[row] : a.n;
    long long T = 64;
    while (T < 2 * cap) T <<= 1;
    if (T > a.slab_T) T = a.slab_T;
    int4* t4 = reinterpret_cast<int4*>(table);
    for (long long s = t; s < T / 4; s += 1024) t4[s] = make_int4(-1, -1, -1, -1);
    if (t == 0) s_lcnt = 0;
    __syncthreads();
    int cnt = 0;
    const GKeys K{table};
    auto f = [&](int key, int) {
      bool ins;
      probe(K, (unsigned)(T - 1), key, ins);
      cnt += ins;
    };
    if (a.flat) {
      for_each_product_block<false, false, int, 1024>(a.a_rpt, a.a_col, nullptr, a.b_rpt, a.b_col, nullptr, true, row,
                                                      t, &s_bf, ws, f, NoStop{});
    } else {
      products<false, false, int, 1024>(false, a.a_rpt, a.a_col, nullptr, a.b_rpt, a.b_col, nullptr, row, t, 1024,
                                        a.vw_log2, f, NoStop{}, a.long_len, &s_lcnt);
      if (a.long_len > 0)
        for_long_products<false, false, int>(a.a_rpt, a.a_col, nullptr, a.b_rpt, a.b_col, nullptr, true, row, t, 1024,
                                             a.long_len, s_list, &s_lcnt, &s_bf, f, NoStop{});
    }
    const long long tot = Grp<1024>::sum(cnt, ws);
    if (t == 0) a.c_cnt[row] = tot;
    __syncthreads();
  }
}

template <int T, int TPR, int BS, bool OPT>
cudaError_t launch_sym(cudaStream_t s, const SymArgs& a) {
  constexpr int RPB = BS / TPR;
  constexpr int smem = RPB * T * 4;
  static_assert(smem <= kSmemLimit - 1024, "symbolic table too large");
  static PerDevice configured;
  auto& cfg = configured.here();
  if (!cfg.load()) {
    cudaError_t e = cudaFuncSetAttribute(k_sym_smem<T, TPR, BS, OPT>,
                                         cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    if (e != cudaSuccess) return e;
    cfg.store(1);
  }
  SymArgs b = a;
  const int max_vw = TPR < 32 ? TPR : 32;
  while ((1 << b.vw_log2) > max_vw) --b.vw_log2;
  const long long grid = (a.nrows + RPB - 1) / RPB;
  k_sym_smem<T, TPR, BS, OPT><<<(unsigned)grid, BS, smem, s>>>(b);
  return cudaGetLastError();
}

// Table slots of group I's hash kernel: kSymTableFactor x the Table-I size (load <= 1/(2 factor))
// where the CTA's tables stay within 64 KB; the optimistic group keeps its fill-limited table.
#ifndef SPG_SYM_TF
#define SPG_SYM_TF 1
#endif
constexpr int kSymTableFactor = SPG_SYM_TF;
template <int I>
constexpr int sym_table() {
  constexpr int T = kSymGroups[I].T, RPB = kSymGroups[I].BS / kSymGroups[I].TPR;
  return (I != kSymOptimistic && RPB * T * kSymTableFactor * 4 <= 64 * 1024) ? T * kSymTableFactor : T;
}

}  // namespace

cudaError_t launch_symbolic_group(cudaStream_t s, int group, const SymArgs& a, int /*num_sms*/) {
  if (a.nrows <= 0) return cudaSuccess;
  switch (group) {
#define SPG_G(I)                                                                              \
  case I:                                                                                     \
    return launch_sym<sym_table<I>(), kSymGroups[I].TPR, kSymGroups[I].BS, (I == kSymOptimistic)>(s, a);
    SPG_G(0) SPG_G(1) SPG_G(2) SPG_G(3) SPG_G(4) SPG_G(5) SPG_G(6) SPG_G(7) SPG_G(8) SPG_G(9) SPG_G(10)
#undef SPG_G
    default: return cudaErrorInvalidValue;
  }
}

cudaError_t launch_symbolic_global(cudaStream_t s, const SymArgs& a, int grid) {
  if (grid <= 0) return cudaSuccess;
  SymArgs b = a;
  if (b.vw_log2 > 5) b.vw_log2 = 5;
  k_sym_global<<<grid, 1024, 0, s>>>(b);
  return cudaGetLastError();
}

}  // namespace spg
