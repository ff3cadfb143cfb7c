// kernels_numeric.cu — step (7) of PAPER.md:80, §III-C: per group of
// rows (grouped by nnz_i in step 6), three phases per row:
//   (a) accumulate: Alg. 5 on the key table plus "another table for the calculation of
//       values" — value slot += a_ik * b_kj in the working precision;
//   (b) gather the non-empty entries;
//   (c) sort by column and write to C at rpt_C[i] + rank.
// All three stay in shared memory when the table fits (PAPER.md:173 last sentence); rows
// above the largest shared-memory group use a per-CTA global-memory slab.
//
// B200 deviation in (b)/(c): the paper's rank sort compares every entry with
// every other (O(nnz_i^2) per row).  Here the gather scatters entries into NB = T/4 buckets
// of the row's column range [lo, hi] (lo/hi tracked with shared atomics at insertion), and
// each entry's rank = start of its bucket + number of smaller keys in the same bucket — the
// paper's comparison rank restricted to the bucket.  Keys are distinct, so the output is
// identical to any correct sort.
#include <climits>

#include "spgemm_internal.cuh"

namespace spg {

namespace {

template <typename VT>
__device__ __forceinline__ void add_value(VT* p, VT v) { atomicAdd(p, v); }

template <typename VT, int TPR, typename SIdx>
__device__ __forceinline__ void num_row(const NumArgs& a, bool active, int row, int* K, VT* V, int* Bc,
                                        SIdx* S, unsigned mask, int NB, int* lohi, long long* ws) {
  const int t = Grp<TPR>::lane();
  const unsigned T = mask + 1;
  // (0) init: keys <- -1 (Alg. 5 precondition), values <- 0
  for (unsigned s = t; s < T; s += TPR) { K[s] = -1; V[s] = VT(0); }
  if (t == 0) { lohi[0] = INT_MAX; lohi[1] = -1; }
  Grp<TPR>::sync();

  // (a) accumulate
  if (active) {
    const VT* __restrict__ av = static_cast<const VT*>(a.a_val);
    const VT* __restrict__ bv = static_cast<const VT*>(a.b_val);
    const long long a0 = a.a_rpt[row], a1 = a.a_rpt[row + 1];
    const int vwl = a.vw_log2;
    const int vw = 1 << vwl, sub = t >> vwl, lane = t & (vw - 1), nsub = TPR >> vwl;
    for (long long j = a0 + sub; j < a1; j += nsub) {
      const int kk = __ldg(a.a_col + j);
      const VT aik = av[j];
      const long long b0 = __ldg(a.b_rpt + kk), b1 = __ldg(a.b_rpt + kk + 1);
      for (long long q = b0 + lane; q < b1; q += vw) {
        const int key = __ldg(a.b_col + q);
        const VT prod = aik * bv[q];  // value <- a_ik b_kj (Alg. 1)
        bool ins;
        const unsigned s = hash_slot(K, mask, key, ins);
        if (ins) { atomicMin(&lohi[0], key); atomicMax(&lohi[1], key); }
        add_value(V + s, prod);
      }
    }
  }
  Grp<TPR>::sync();

  // (b) gather: bucket histogram over the column range
  const int lo = lohi[0], hi = lohi[1];
  int shift = 0, nb = 0;
  if (hi >= lo) {
    const unsigned R = (unsigned)(hi - lo);
    while ((R >> shift) >= (unsigned)NB) ++shift;
    nb = (int)(R >> shift) + 1;
  }
  for (int b = t; b <= nb; b += TPR) Bc[b] = 0;
  Grp<TPR>::sync();
  for (unsigned s = t; s < T; s += TPR) {
    const int key = K[s];
    if (key >= 0) atomicAdd(&Bc[1 + ((key - lo) >> shift)], 1);
  }
  Grp<TPR>::sync();
  long long n_total;
  {
    const int per = (nb + TPR - 1) / TPR;
    const int b0 = 1 + t * per;
    const int b1 = min(nb + 1, b0 + per);
    long long loc = 0;
    for (int b = b0; b < b1; ++b) loc += Bc[b];
    long long run = Grp<TPR>::excl_scan(loc, &n_total, ws);
    for (int b = b0; b < b1; ++b) { const int c = Bc[b]; Bc[b] = (int)run; run += c; }
  }
  Grp<TPR>::sync();
  for (unsigned s = t; s < T; s += TPR) {
    const int key = K[s];
    if (key >= 0) S[atomicAdd(&Bc[1 + ((key - lo) >> shift)], 1)] = (SIdx)s;
  }
  Grp<TPR>::sync();

  // (c) rank = bucket start + #smaller keys in the bucket; write C
  if (active) {
    const long long c0 = a.c_rpt[row];
    const long long cn = a.c_rpt[row + 1] - c0;
    if (t == 0 && cn != n_total) atomicOr(a.err_flags, 2);
    VT* __restrict__ cv = static_cast<VT*>(a.c_val);
    for (long long p = t; p < n_total; p += TPR) {
      const unsigned s = S[p];
      const int key = K[s];
      const int b = (key - lo) >> shift;
      const int st = Bc[b], en = Bc[b + 1];
      int r = st;
      for (int q = st; q < en; ++q) r += (K[S[q]] < key);
      if (r < cn) {
        a.c_col[c0 + r] = key;
        cv[c0 + r] = V[s];
      }
    }
  }
  Grp<TPR>::sync();
}

template <typename VT, int T, int TPR, int BS, long long UPPER>
__global__ __launch_bounds__(BS) void k_num_smem(NumArgs a) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  __shared__ long long ws[33];
  constexpr int RPB = BS / TPR;
  __shared__ int s_lohi[2 * RPB];
  constexpr int NB = num_nbuckets(T);
  constexpr int RB = num_row_bytes<VT>(T, UPPER);
  const int g = threadIdx.x / TPR;
  unsigned char* base = smem_raw + g * RB;
  VT* V = reinterpret_cast<VT*>(base);
  int* K = reinterpret_cast<int*>(base + T * sizeof(VT));
  int* Bc = K + T;
  uint16_t* S = reinterpret_cast<uint16_t*>(Bc + NB + 1);
  const long long ridx = (long long)blockIdx.x * RPB + g;
  const bool active = ridx < a.nrows;
  const int row = active ? a.rows[ridx] : 0;
  num_row<VT, TPR, uint16_t>(a, active, row, K, V, Bc, S, T - 1, NB, s_lohi + 2 * g, ws);
}

template <typename VT>
__global__ __launch_bounds__(1024) void k_num_global(NumArgs a) {
  __shared__ long long ws[33];
  __shared__ int s_lohi[2];
  unsigned char* slab = static_cast<unsigned char*>(a.slab) + (long long)blockIdx.x * a.slab_stride;
  VT* V = reinterpret_cast<VT*>(slab);
  int* K = reinterpret_cast<int*>(V + a.slab_T);
  int* Bc = K + a.slab_T;
  int* S = Bc + a.slab_T / 4 + 1;
  for (long long i = blockIdx.x; i < a.nrows; i += gridDim.x) {
    const int row = a.rows[i];
    const long long n = a.c_rpt[row + 1] - a.c_rpt[row];
    long long T = 64;
    while (T < 2 * n) T <<= 1;
    if (T > a.slab_T) T = a.slab_T;
    num_row<VT, 1024, int>(a, true, row, K, V, Bc, S, (unsigned)(T - 1), (int)(T / 4), s_lohi, ws);
  }
}

template <typename VT, int T, int TPR, int BS, long long UPPER>
cudaError_t launch_num(cudaStream_t s, const NumArgs& a) {
  constexpr int RPB = BS / TPR;
  constexpr int smem = RPB * num_row_bytes<VT>(T, UPPER);
  static_assert(smem + 33 * 8 + 8 * RPB <= kSmemLimit, "numeric table too large");
  static bool configured = false;
  if (!configured) {
    cudaError_t e = cudaFuncSetAttribute(k_num_smem<VT, T, TPR, BS, UPPER>,
                                         cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    if (e != cudaSuccess) return e;
    configured = true;
  }
  NumArgs b = a;
  const int max_vw = TPR < 32 ? TPR : 32;
  while ((1 << b.vw_log2) > max_vw) --b.vw_log2;
  const long long grid = (a.nrows + RPB - 1) / RPB;
  k_num_smem<VT, T, TPR, BS, UPPER><<<(unsigned)grid, BS, smem, s>>>(b);
  return cudaGetLastError();
}

template <typename VT>
cudaError_t launch_num_group(cudaStream_t s, int group, const NumArgs& a) {
  switch (group) {
#define SPG_G(I)                                                                                      \
  case I:                                                                                             \
    return launch_num<VT, kNumGroups[I].T, kNumGroups[I].TPR, kNumGroups[I].BS, kNumGroups[I].upper>(s, a);
    SPG_G(0) SPG_G(1) SPG_G(2) SPG_G(3) SPG_G(4) SPG_G(5) SPG_G(6) SPG_G(7) SPG_G(8) SPG_G(9)
#undef SPG_G
    default: return cudaErrorInvalidValue;
  }
}

}  // namespace

cudaError_t launch_numeric_group(cudaStream_t s, int group, bool fp64, const NumArgs& a) {
  if (a.nrows <= 0) return cudaSuccess;
  return fp64 ? launch_num_group<double>(s, group, a) : launch_num_group<float>(s, group, a);
}

cudaError_t launch_numeric_global(cudaStream_t s, bool fp64, const NumArgs& a, int grid) {
  if (grid <= 0 || a.nrows <= 0) return cudaSuccess;
  NumArgs b = a;
  if (b.vw_log2 > 5) b.vw_log2 = 5;
  if (fp64) k_num_global<double><<<grid, 1024, 0, s>>>(b);
  else k_num_global<float><<<grid, 1024, 0, s>>>(b);
  return cudaGetLastError();
}

}  // namespace spg
