// kernels_rankacc.cu — numeric step (7) for CTA-per-row groups of wide-span (graph) rows:
// accumulation into a table indexed by the RANK of the column in the row (B200 addition,
// DESIGN.md §5.8).
//
// The paper's numeric phase inserts every product's column into a hash table
// (Alg. 5), adds the value into a parallel value table, then gathers the occupied slots and sorts
// them by a comparison rank.  Its final position is rank(key) = #distinct columns of row i below
// key.  For rows of C whose column span is wide and sparse (power-law graphs: R-MAT, webbase —
// products ~ output entries, so the hash tables are nearly all fixed cost) this kernel computes
// that rank FIRST, from a two-level bitmap of the row's columns over its exact span [lo_i, hi_i]
// (from step (1)), and uses it as a collision-free, order-preserving hash:
//
//   (i)   metadata: the row's A non-zeros (<= TPR), one per thread: col_A, val_A, rpt_B pair;
//         block scan of the B-row lengths (Alg. 3/4's product enumeration, flattened);
//   (ii)  gather: thread t takes products t, t+TPR, ... (<= KP of them, held in registers; all
//         gathers of b_col/b_val issued before use) and sets level-1 bit (key-lo)>>5 — "32-column
//         block is non-empty" — with a shared atomicOr;
//   (iii) prefix popcount of level 1 -> compact index of every non-empty block;
//   (iv)  each product sets its bit in the level-2 word of its block;
//   (v)   prefix popcount of level 2 -> rank(key) = pre2[b] + popc(fine[b] & below(key));
//   (vi)  vals[rank] += a_ik * b_kj (shared atomic add, working precision),
//         keys[rank] = key (idempotent store);
//   (vii) the row is now compact and sorted: coalesced write of keys/vals to C.
//
// No probing, no -1 initialisation of a 2x-oversized table, no compaction or sort pass; O(n_prod
// + R_i/1024) work with a handful of CTA barriers.  Rows with more than TPR A non-zeros or more
// than KP*TPR products walk the products with the chunked block loop once per pass (re-gathering;
// the result is identical).  The paper's hash path (kernels_numeric.cu) stays for rows without a
// column span (range hash disabled) and as the forced-path reference.
#include <climits>

#include "spgemm_internal.cuh"

namespace spg {

namespace {

struct NoStopR {
  __device__ __forceinline__ bool operator()() const { return false; }
};

// 32-bit CTA exclusive scan with one barrier; ws32 holds >= 32 ints and must not be reused by the
// next scan before a barrier separates them (callers alternate two buffers).
template <int TPR>
__device__ __forceinline__ int cta_scan32(int v, int* total, int* ws32) {
  constexpr int NW = TPR / 32;
  const int l = threadIdx.x & 31, w = threadIdx.x >> 5;
  int x = v;
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    const int y = __shfl_up_sync(0xffffffffu, x, d);
    if (l >= d) x += y;
  }
  if (l == 31) ws32[w] = x;
  __syncthreads();
  int s = l < NW ? ws32[l] : 0;
#pragma unroll
  for (int d = 1; d < NW; d <<= 1) {
    const int y = __shfl_up_sync(0xffffffffu, s, d);
    if (l >= d) s += y;
  }
  const int base = __shfl_sync(0xffffffffu, s, (w + 31) & 31);  // inclusive total of warps < w
  *total = __shfl_sync(0xffffffffu, s, NW - 1);
  return (w > 0 ? base : 0) + x - v;
}

// Dynamic shared memory layout (16-byte aligned pieces):
//   vals[UPPER] VT | b0[TPR] i64 | av[TPR] VT | incl[TPR] i32 | keys[UPPER] i32 |
//   fine[UPPER] u32 | l1[L1W] u32 | pre2[UPPER] u16 | p1[L1W] u16
template <typename VT, int TPR, long long UPPER>
struct RankLayout {
  static constexpr int kVals = 0;
  static constexpr int kB0 = align16((int)(UPPER * sizeof(VT)));
  static constexpr int kAv = kB0 + align16(TPR * 8);
  static constexpr int kIncl = kAv + align16(TPR * (int)sizeof(VT));
  static constexpr int kKeys = kIncl + align16(TPR * 4);
  static constexpr int kFine = kKeys + align16((int)UPPER * 4);
  static constexpr int kL1 = kFine + align16((int)UPPER * 4);
  static __host__ __device__ constexpr int pre2(int l1w) { return kL1 + align16(l1w * 4); }
  static __host__ __device__ constexpr int p1(int l1w) { return pre2(l1w) + align16((int)UPPER * 2); }
  static __host__ __device__ constexpr int bytes(int l1w) { return p1(l1w) + align16(l1w * 2); }
};

template <typename VT, int TPR, long long UPPER, int KP>
__global__ __launch_bounds__(TPR, TPR >= 1024 ? 1 : 2048 / TPR / 2) void k_num_rankacc(NumArgs a) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  using L = RankLayout<VT, TPR, UPPER>;
  __shared__ int ws32[2][32];
  __shared__ long long ws64[33];
  VT* vals = reinterpret_cast<VT*>(smem_raw + L::kVals);
  long long* sb0 = reinterpret_cast<long long*>(smem_raw + L::kB0);
  VT* sav = reinterpret_cast<VT*>(smem_raw + L::kAv);
  int* sincl = reinterpret_cast<int*>(smem_raw + L::kIncl);
  int* keys = reinterpret_cast<int*>(smem_raw + L::kKeys);
  unsigned* fine = reinterpret_cast<unsigned*>(smem_raw + L::kFine);
  unsigned* l1 = reinterpret_cast<unsigned*>(smem_raw + L::kL1);
  uint16_t* pre2 = reinterpret_cast<uint16_t*>(smem_raw + L::pre2(a.l1_words));
  uint16_t* p1 = reinterpret_cast<uint16_t*>(smem_raw + L::p1(a.l1_words));
  // the chunked fallback walk reuses b0/av/incl through the BlockFlat view (same field order)
  static_assert(sizeof(BlockFlat<VT, TPR>) <= (size_t)(L::kKeys - L::kB0) + 64, "block-flat view");

  const VT* __restrict__ av_g = static_cast<const VT*>(a.a_val);
  const VT* __restrict__ bv_g = static_cast<const VT*>(a.b_val);
  const int32_t* __restrict__ bc_g = a.b_col;
  const int t = threadIdx.x;
  const int row = a.rows[blockIdx.x];
  const long long a0 = __ldg(a.a_rpt + row);
  const int na = (int)(__ldg(a.a_rpt + row + 1) - a0);
  const long long c0 = a.c_rpt[row];
  const int cn = (int)(a.c_rpt[row + 1] - c0);
  const int2 rr = __ldg(a.rlohi + row);
  const int lo = rr.x;
  const int W1 = rr.y >= rr.x ? (int)(((unsigned)(rr.y - rr.x)) >> 10) + 1 : 0;  // CTA-uniform
  for (int w = t; w < W1; w += TPR) l1[w] = 0u;

  // (i) metadata of the first TPR A non-zeros + scan of their B-row lengths
  int len = 0;
  if (t < na) {
    const int kk = __ldg(a.a_col + a0 + t);
    const long long b0 = __ldg(a.b_rpt + kk);
    len = (int)(__ldg(a.b_rpt + kk + 1) - b0);
    sb0[t] = b0;
    sav[t] = __ldg(av_g + a0 + t);
  }
  int P;
  const int ex = cta_scan32<TPR>(t < na ? len : 0, &P, ws32[0]);
  if (t < na) sincl[t] = ex + len;
  __syncthreads();
  const bool fast = na <= TPR && P <= KP * TPR;  // CTA-uniform

  int key[KP];
  VT val[KP];
  auto locate = [&](int p, int& e, long long& q) {  // product p -> its A entry e and B position q
    int l = 0, h = min(na, TPR) - 1;
    while (l < h) {
      const int mid = (l + h) >> 1;
      if (sincl[mid] <= p) l = mid + 1; else h = mid;
    }
    e = l;
    q = sb0[l] + (p - (l ? sincl[l - 1] : 0));
  };
  auto set_l1 = [&](int k) {
    const unsigned d = (unsigned)(k - lo);
    atomicOr(l1 + (d >> 10), 1u << ((d >> 5) & 31));
  };
  auto blk_of = [&](unsigned d) {
    const unsigned w = d >> 10, bit = (d >> 5) & 31;
    return (int)p1[w] + __popc(l1[w] & ((1u << bit) - 1u));
  };
  auto set_fine = [&](int k) {
    const unsigned d = (unsigned)(k - lo);
    atomicOr(fine + blk_of(d), 1u << (d & 31));
  };
  auto accumulate = [&](int k, VT v) {
    const unsigned d = (unsigned)(k - lo);
    const int b = blk_of(d);
    const int r = (int)pre2[b] + __popc(fine[b] & ((1u << (d & 31)) - 1u));
    atomicAdd(vals + r, v);
    keys[r] = k;
  };
  BlockFlat<VT, TPR>* bf = reinterpret_cast<BlockFlat<VT, TPR>*>(sb0);
  auto walk = [&](auto&& f) {  // slow path: chunked block loop over all products (re-gathers)
    for_each_product_block<true, false, VT, TPR>(a.a_rpt, a.a_col, av_g, a.b_rpt, bc_g, bv_g, true, row, t, bf,
                                                 ws64, f, NoStopR{});
  };

  // (ii) gather + level 1
  if (fast) {
#pragma unroll
    for (int u = 0; u < KP; ++u) {
      const int p = t + u * TPR;
      key[u] = -1;
      if (p < P) {
        int e;
        long long q;
        locate(p, e, q);
        key[u] = __ldg(bc_g + q);
        val[u] = sav[e] * __ldg(bv_g + q);
      }
    }
#pragma unroll
    for (int u = 0; u < KP; ++u)
      if (key[u] >= 0) set_l1(key[u]);
  } else {
    __syncthreads();  // the walk overwrites b0/av/incl
    walk([&](int k, VT) { set_l1(k); });
  }
  __syncthreads();
  // (iii) compact index of the non-empty 32-column blocks
  int nb;
  {
    const int per = (W1 + TPR - 1) / TPR;
    const int w0 = min(W1, t * per), w1 = min(W1, w0 + per);
    int loc = 0;
    for (int w = w0; w < w1; ++w) loc += __popc(l1[w]);
    int run = cta_scan32<TPR>(loc, &nb, ws32[1]);
    for (int w = w0; w < w1; ++w) { p1[w] = (uint16_t)run; run += __popc(l1[w]); }
  }
  for (int b = t; b < nb; b += TPR) fine[b] = 0u;
  __syncthreads();
  // (iv) level 2
  if (fast) {
#pragma unroll
    for (int u = 0; u < KP; ++u)
      if (key[u] >= 0) set_fine(key[u]);
  } else {
    walk([&](int k, VT) { set_fine(k); });
  }
  __syncthreads();
  // (v) rank of every block's first key
  int n_total;
  {
    const int per = (nb + TPR - 1) / TPR;
    const int b0 = min(nb, t * per), b1 = min(nb, b0 + per);
    int loc = 0;
    for (int b = b0; b < b1; ++b) loc += __popc(fine[b]);
    int run = cta_scan32<TPR>(loc, &n_total, ws32[0]);
    for (int b = b0; b < b1; ++b) { pre2[b] = (uint16_t)run; run += __popc(fine[b]); }
  }
  if (t == 0 && n_total != cn) atomicOr(a.err_flags, 2);
  const int nw = min(n_total, cn);
  for (int r = t; r < nw; r += TPR) vals[r] = VT(0);
  __syncthreads();
  // (vi) accumulate at the rank
  if (fast) {
#pragma unroll
    for (int u = 0; u < KP; ++u)
      if (key[u] >= 0) accumulate(key[u], val[u]);
  } else {
    walk([&](int k, VT v) { accumulate(k, v); });
  }
  __syncthreads();
  // (vii) sorted, compact row -> C (coalesced)
  int32_t* __restrict__ cc = a.c_col + c0;
  VT* __restrict__ cv = static_cast<VT*>(a.c_val) + c0;
  for (int r = t; r < nw; r += TPR) {
    cc[r] = keys[r];
    cv[r] = vals[r];
  }
}

template <typename VT, int TPR, long long UPPER>
cudaError_t launch_rankacc_k(cudaStream_t s, const NumArgs& a) {
  constexpr int KP = 8;
  using L = RankLayout<VT, TPR, UPPER>;
  const int smem = L::bytes(a.l1_words);
  static int configured = 0;
  if (smem > configured) {
    cudaError_t e = cudaFuncSetAttribute(k_num_rankacc<VT, TPR, UPPER, KP>,
                                         cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    if (e != cudaSuccess) return e;
    configured = smem;
  }
  k_num_rankacc<VT, TPR, UPPER, KP><<<(unsigned)a.nrows, TPR, smem, s>>>(a);
  return cudaGetLastError();
}

template <typename VT>
cudaError_t launch_rankacc_v(cudaStream_t s, int group, const NumArgs& a) {
  switch (group) {
#define SPG_G(I)                                                                                  \
  case I:                                                                                         \
    return launch_rankacc_k<VT, kNumGroups[I].TPR, kNumGroups[I].upper>(s, a);
    SPG_G(4) SPG_G(5) SPG_G(6) SPG_G(7) SPG_G(8) SPG_G(9)
#undef SPG_G
    default: return cudaErrorInvalidValue;
  }
}

}  // namespace

int rankacc_smem_bytes(int group, bool fp64, int l1_words) {
  switch (group) {
#define SPG_G(I)                                                                                              \
  case I:                                                                                                     \
    return fp64 ? RankLayout<double, kNumGroups[I].TPR, kNumGroups[I].upper>::bytes(l1_words) + 1400         \
                : RankLayout<float, kNumGroups[I].TPR, kNumGroups[I].upper>::bytes(l1_words) + 1400;
    SPG_G(4) SPG_G(5) SPG_G(6) SPG_G(7) SPG_G(8) SPG_G(9)
#undef SPG_G
    default: return INT_MAX;
  }
}

cudaError_t launch_numeric_rankacc(cudaStream_t s, int group, bool fp64, const NumArgs& a) {
  if (a.nrows <= 0) return cudaSuccess;
  return fp64 ? launch_rankacc_v<double>(s, group, a) : launch_rankacc_v<float>(s, group, a);
}

}  // namespace spg
