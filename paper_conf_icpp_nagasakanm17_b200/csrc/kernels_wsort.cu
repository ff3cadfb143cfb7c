// kernels_wsort.cu — warp-per-row kernels that ORDER a row's products in registers (B200
// addition) for rows of up to 32*ITEMS products: symbolic count (step (3)) and
// numeric accumulate + gather + sort + write (step (7)).
//
// The paper's small and medium rows (PWARP/ROW and TB/ROW) insert every product
// into a shared-memory hash table (Alg. 5), then gather and rank-sort the table.
// Here one warp owns the row and holds its products in registers, ITEMS per lane in blocked order
// (element i = lane*ITEMS + item): a bitonic network — register compare-exchanges for strides
// below ITEMS, shuffles above — sorts the (column, value) pairs; equal columns are then adjacent, the
// first of each run is the row's entry (the distinct-key count of PAPER.md:153 in the symbolic
// phase), its run is summed in the working precision and its position is the number
// of entries before it (the rank of PAPER.md:173).  No table initialisation, no probing, no CTA
// barriers and no shared memory in the symbolic kernel; the numeric kernel stages the sorted row in
// warp-private shared memory for the run sums and a coalesced write of the compacted row.
#include <climits>

#include "spgemm_internal.cuh"

namespace spg {

namespace {

constexpr unsigned kWFull = 0xffffffffu;
constexpr int kWarpsPerBlock = 4;

// Products of `row` into key[it] / val[it] for element lane*ITEMS + it (Alg. 1 order; INT_MAX past
// the row's n_prod_i).  A entries are taken 32 at a time (one per lane); a product finds its
// entry by a shuffle binary search over the chunk's inclusive length scan.  Returns n_prod_i, or
// -1 when the row has more than 32*ITEMS products (the caller routes such rows elsewhere).
template <bool NUM, typename VT, int ITEMS>
__device__ __forceinline__ int wsort_load(const int64_t* __restrict__ a_rpt, const int32_t* __restrict__ a_col,
                                          const VT* __restrict__ a_val, const int64_t* __restrict__ b_rpt,
                                          const int32_t* __restrict__ b_col, const VT* __restrict__ b_val, int row,
                                          int lane, int (&key)[ITEMS], VT (&val)[ITEMS]) {
  const long long a0 = __ldg(a_rpt + row), a1 = __ldg(a_rpt + row + 1);
#pragma unroll
  for (int it = 0; it < ITEMS; ++it) {
    key[it] = INT_MAX;
    if (NUM) val[it] = VT(0);
  }
  int base = 0;  // products before this chunk
  for (long long c = a0; c < a1; c += 32) {  // warp-uniform
    long long b0 = 0;
    int len = 0;
    VT av = VT(0);
    if (c + lane < a1) {
      const int kk = __ldg(a_col + c + lane);
      if (NUM) av = __ldg(a_val + c + lane);
      b0 = __ldg(b_rpt + kk);
      len = (int)(__ldg(b_rpt + kk + 1) - b0);
    }
    int incl = len;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
      const int y = __shfl_up_sync(kWFull, incl, d);
      if (lane >= d) incl += y;
    }
    const int tot = __shfl_sync(kWFull, incl, 31);
    if (base + tot > 32 * ITEMS) return -1;  // warp-uniform
#pragma unroll
    for (int it = 0; it < ITEMS; ++it) {
      const int p = lane * ITEMS + it - base;  // product index within the chunk
      int e = 0;
#pragma unroll
      for (int st = 16; st > 0; st >>= 1)
        if (__shfl_sync(kWFull, incl, e + st - 1) <= p) e += st;
      const int ex = __shfl_sync(kWFull, incl - len, e & 31);
      const long long eb = __shfl_sync(kWFull, b0, e & 31);
      const VT ea = NUM ? __shfl_sync(kWFull, av, e & 31) : VT(0);
      if (p >= 0 && p < tot) {
        const long long q = eb + (p - ex);
        key[it] = __ldg(b_col + q);
        if (NUM) val[it] = ea * __ldg(b_val + q);
      }
    }
    base += tot;
  }
  return base;
}

// Ascending bitonic sort of the warp's 32*ITEMS (key, val) pairs, blocked layout.
template <bool NUM, typename VT, int ITEMS>
__device__ __forceinline__ void wsort_sort(int lane, int (&key)[ITEMS], VT (&val)[ITEMS]) {
  constexpr int N = 32 * ITEMS;
#pragma unroll
  for (int k = 2; k <= N; k <<= 1) {
#pragma unroll
    for (int j = k >> 1; j > 0; j >>= 1) {
      if (j < ITEMS) {  // partner in this lane
#pragma unroll
        for (int it = 0; it < ITEMS; ++it) {
          const int pt = it ^ j;
          if (pt > it) {
            const bool up = ((lane * ITEMS + it) & k) == 0;
            if ((key[it] > key[pt]) == up && key[it] != key[pt]) {
              const int tk = key[it]; key[it] = key[pt]; key[pt] = tk;
              if (NUM) { const VT tv = val[it]; val[it] = val[pt]; val[pt] = tv; }
            }
          }
        }
      } else {  // partner lane = lane ^ (j / ITEMS), same item
#pragma unroll
        for (int it = 0; it < ITEMS; ++it) {
          const int ok = __shfl_xor_sync(kWFull, key[it], j / ITEMS);
          const VT ov = NUM ? __shfl_xor_sync(kWFull, val[it], j / ITEMS) : VT(0);
          const int i = lane * ITEMS + it;
          const bool up = (i & k) == 0, lower = (i & j) == 0;
          const bool take = up == lower ? ok < key[it] : ok > key[it];
          if (take) {
            key[it] = ok;
            if (NUM) val[it] = ov;
          }
        }
      }
    }
  }
}

// Head flags (first of a run of equal keys) of this lane's ITEMS sorted elements; returns the mask.
template <int ITEMS>
__device__ __forceinline__ unsigned wsort_heads(int lane, const int (&key)[ITEMS]) {
  const int prev_last = __shfl_up_sync(kWFull, key[ITEMS - 1], 1);
  unsigned hm = 0;
#pragma unroll
  for (int it = 0; it < ITEMS; ++it) {
    const int prev = it ? key[it - 1] : prev_last;
    if (key[it] != INT_MAX && ((lane == 0 && it == 0) || prev != key[it])) hm |= 1u << it;
  }
  return hm;
}

template <int ITEMS>
__global__ __launch_bounds__(32 * kWarpsPerBlock) void k_sym_wsort(SymArgs a) {
  const long long w = ((long long)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int lane = threadIdx.x & 31;
  if (w >= a.nrows) return;  // warp-uniform
  const int row = __ldg(a.rows + w);
  int key[ITEMS];
  int dummy[ITEMS];
  const int np = wsort_load<false, int, ITEMS>(a.a_rpt, a.a_col, nullptr, a.b_rpt, a.b_col, nullptr, row, lane, key,
                                               dummy);
  if (np < 0) {  // more products than the group bound: inconsistent grouping
    if (lane == 0) atomicOr(a.err_flags, 1);
    return;
  }
  wsort_sort<false, int, ITEMS>(lane, key, dummy);
  const int n = __reduce_add_sync(kWFull, __popc(wsort_heads<ITEMS>(lane, key)));
  if (lane == 0) a.c_cnt[row] = n;
}

// Warp-private staging of the sorted row (swizzled: element i at i + i/32).
template <typename VT, int ITEMS>
struct WsortStage {
  static constexpr int N = 32 * ITEMS;
  int k[N + N / 32];
  VT v[N + N / 32];
};

template <typename VT, int ITEMS>
__global__ __launch_bounds__(32 * kWarpsPerBlock) void k_num_wsort(NumArgs a) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  using St = WsortStage<VT, ITEMS>;
  constexpr int N = St::N;
  St* stg = reinterpret_cast<St*>(smem_raw) + (threadIdx.x >> 5);
  const long long w = ((long long)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int lane = threadIdx.x & 31;
  if (w >= a.nrows) return;  // warp-uniform
  const int row = __ldg(a.rows + w);
  int key[ITEMS];
  VT val[ITEMS];
  const int np = wsort_load<true, VT, ITEMS>(a.a_rpt, a.a_col, static_cast<const VT*>(a.a_val), a.b_rpt, a.b_col,
                                             static_cast<const VT*>(a.b_val), row, lane, key, val);
  const long long c0 = a.c_rpt[row];
  const int cn = (int)(a.c_rpt[row + 1] - c0);
  if (np < 0) {
    if (lane == 0) atomicOr(a.err_flags, 2);
    return;
  }
  wsort_sort<true, VT, ITEMS>(lane, key, val);
  const unsigned hm = wsort_heads<ITEMS>(lane, key);
  // stage the sorted row for the run sums (runs may cross lanes)
#pragma unroll
  for (int it = 0; it < ITEMS; ++it) {
    const int i = lane * ITEMS + it;
    stg->k[i + (i >> 5)] = key[it];
    stg->v[i + (i >> 5)] = val[it];
  }
  int nh = __popc(hm);
  int off = nh;
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    const int y = __shfl_up_sync(kWFull, off, d);
    if (lane >= d) off += y;
  }
  const int total = __shfl_sync(kWFull, off, 31);
  off -= nh;  // entries before this lane's first element
  if (total != cn) {
    if (lane == 0) atomicOr(a.err_flags, 2);
    return;
  }
  __syncwarp();
  // each head sums its run (in sorted order) and keeps (output position, key, sum) in registers
  int opos[ITEMS];
#pragma unroll
  for (int it = 0; it < ITEMS; ++it) {
    opos[it] = -1;
    if (hm & (1u << it)) {
      const int i = lane * ITEMS + it;
      VT s = val[it];
      for (int q = i + 1; q < np; ++q) {
        const int k2 = stg->k[q + (q >> 5)];
        if (k2 != key[it]) break;
        s += stg->v[q + (q >> 5)];
      }
      val[it] = s;
      opos[it] = off++;
    }
  }
  __syncwarp();
#pragma unroll
  for (int it = 0; it < ITEMS; ++it)
    if (opos[it] >= 0) {
      stg->k[opos[it] + (opos[it] >> 5)] = key[it];
      stg->v[opos[it] + (opos[it] >> 5)] = val[it];
    }
  __syncwarp();
  int32_t* __restrict__ cc = a.c_col + c0;
  VT* __restrict__ cv = static_cast<VT*>(a.c_val) + c0;
  for (int o = lane; o < cn; o += 32) {
    cc[o] = stg->k[o + (o >> 5)];
    cv[o] = stg->v[o + (o >> 5)];
  }
}

template <int ITEMS>
cudaError_t launch_sym_wsort_i(cudaStream_t s, const SymArgs& a) {
  const long long threads = a.nrows * 32;
  k_sym_wsort<ITEMS><<<(unsigned)((threads + 32 * kWarpsPerBlock - 1) / (32 * kWarpsPerBlock)), 32 * kWarpsPerBlock, 0,
                       s>>>(a);
  return cudaGetLastError();
}

template <typename VT, int ITEMS>
cudaError_t launch_num_wsort_i(cudaStream_t s, const NumArgs& a) {
  constexpr int smem = (int)sizeof(WsortStage<VT, ITEMS>) * kWarpsPerBlock;
  static PerDevice cache;
  auto& c = cache.here();
  if (smem > 48 * 1024 && smem > c.load()) {
    cudaError_t e = cudaFuncSetAttribute(k_num_wsort<VT, ITEMS>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    if (e != cudaSuccess) return e;
    c.store(smem);
  }
  const long long threads = a.nrows * 32;
  k_num_wsort<VT, ITEMS><<<(unsigned)((threads + 32 * kWarpsPerBlock - 1) / (32 * kWarpsPerBlock)),
                           32 * kWarpsPerBlock, smem, s>>>(a);
  return cudaGetLastError();
}

}  // namespace

// Symbolic groups served: 2 (n_prod <= 128: 4 per lane), 3 (<= 256: 8), 4 (<= 512: 16), 5 (<= 1024: 32).
int wsort_max_group() { return 5; }

cudaError_t launch_symbolic_wsort(cudaStream_t s, int sym_group, const SymArgs& a) {
  if (a.nrows <= 0) return cudaSuccess;
  static_assert(kSymGroups[2].upper == 128 && kSymGroups[5].upper == 1024, "wsort capacities");
  switch (sym_group) {
    case 2: return launch_sym_wsort_i<4>(s, a);
    case 3: return launch_sym_wsort_i<8>(s, a);
    case 4: return launch_sym_wsort_i<16>(s, a);
    case 5: return launch_sym_wsort_i<32>(s, a);
    default: return cudaErrorInvalidValue;
  }
}

cudaError_t launch_numeric_wsort(cudaStream_t s, int sym_group, bool fp64, const NumArgs& a) {
  if (a.nrows <= 0) return cudaSuccess;
  switch (sym_group) {
    case 2: return fp64 ? launch_num_wsort_i<double, 4>(s, a) : launch_num_wsort_i<float, 4>(s, a);
    case 3: return fp64 ? launch_num_wsort_i<double, 8>(s, a) : launch_num_wsort_i<float, 8>(s, a);
    case 4: return fp64 ? launch_num_wsort_i<double, 16>(s, a) : launch_num_wsort_i<float, 16>(s, a);
    case 5: return fp64 ? launch_num_wsort_i<double, 32>(s, a) : launch_num_wsort_i<float, 32>(s, a);
    default: return cudaErrorInvalidValue;
  }
}

}  // namespace spg
