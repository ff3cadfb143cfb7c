// kernels_cluster.cu — cluster-per-row variants (B200 addition to PAPER.md:155, 181): rows whose
// hash table exceeds one SM's shared memory keep it in the distributed shared memory (DSMEM)
// of a thread-block cluster of kCS CTAs on kCS SMs instead of in global memory.
//
// The table of T = kCS * Ts slots is split in kCS contiguous slices, slot h living in CTA
// h / Ts at local index h % Ts; linear probing (Alg. 5) walks across slice boundaries.  Remote
// slots are reached through generic pointers from cluster.map_shared_rank (ATOM.E.CAS /
// ATOM.E.ADD on sm_100a).  All kCS*1024 threads of the cluster share a row: the A non-zeros
// are spread over the whole cluster (for_each_product with a cluster-wide thread index), and
// deferred long B rows are split between the CTAs.
//
//   k_sym_cluster: counts the distinct keys of rows that overflowed the single-CTA optimistic
//     table; a row that finds more than fill_limit keys is recorded again (overflow2) and
//     recounted in a global-memory table (k_sym_global).
//   k_num_cluster: accumulate into the distributed key/value table, then rank with a bitmap
//     over the row's column span in a per-cluster global scratch (prefix popcounts), write C.
#include <cooperative_groups.h>

#include <climits>

#include "spgemm_internal.cuh"

namespace cg = cooperative_groups;

namespace spg {

namespace {

struct NoStop {
  __device__ __forceinline__ bool operator()() const { return false; }
};

// Distributed key table: slice pointers of all CTAs of the cluster (shared array of kCS).
struct CKeys {
  int* const* sl;
  unsigned ls, lm;  // log2(Ts), Ts - 1
  __device__ __forceinline__ int* at(unsigned h) const { return sl[h >> ls] + (h & lm); }
  __device__ __forceinline__ int ld(unsigned h) const { return *(const volatile int*)at(h); }
  __device__ __forceinline__ int cas(unsigned h, int c, int v) const { return atomicCAS(at(h), c, v); }
};

template <typename VT>
struct CVals {
  VT* const* sl;
  unsigned ls, lm;
  __device__ __forceinline__ void add(unsigned h, VT v) const { atomicAdd(sl[h >> ls] + (h & lm), v); }
};

// Rows of the cluster: `rows[i]` for i < nA, then overflow_in[i - nA] for i < nA + *count_in.
__device__ __forceinline__ long long cluster_rows_total(long long nA, const int* count_in) {
  return nA + (count_in ? (long long)*count_in : 0);
}

template <int CS>
__global__ void __launch_bounds__(1024) k_sym_cluster(SymArgs a, const int32_t* rows_in, const int* count_in,
                                                     int32_t* overflow2, int* count2, int fill_limit) {
  extern __shared__ __align__(16) int smem[];
  __shared__ int* s_kp[CS];
  __shared__ int s_list[kLongChunk], s_lcnt;
  __shared__ BlockFlat<int> s_bf;
  __shared__ int s_cnt, s_abort;
  cg::cluster_group cluster = cg::this_cluster();
  const int rank = (int)cluster.block_rank();
  const int t = threadIdx.x;
  constexpr int Ts = kClusterSymSlots;
  if (t < CS) s_kp[t] = cluster.map_shared_rank(smem, t);
  int* cnt0 = cluster.map_shared_rank(&s_cnt, 0);
  const long long nclusters = gridDim.x / CS;
  const long long cid = blockIdx.x / CS;
  const long long nrows = cluster_rows_total(a.nrows, count_in);
  const CKeys K{s_kp, 31 - __clz(Ts), Ts - 1};
  const unsigned mask = CS * Ts - 1;
  for (long long i = cid; i < nrows; i += nclusters) {
    const int row = i < a.nrows ? rows_in[i] : a.overflow_rows[i - a.nrows];
    int4* t4 = reinterpret_cast<int4*>(smem);
    for (int s = t; s < Ts / 4; s += 1024) t4[s] = make_int4(-1, -1, -1, -1);
    if (t == 0) { s_cnt = 0; s_abort = 0; s_lcnt = 0; }
    cluster.sync();
    int mine = 0;
    const unsigned ab = smem_u32(&s_abort);
    auto stop = [ab]() { return lds_s32(ab) != 0; };
    auto f = [&](int key, int) {
      bool ins;
      probe(K, mask, key, ins);
      if (ins) {
        ++mine;
        if (atomicAdd(cnt0, 1) + 1 >= fill_limit) {  // raise every CTA's abort flag
          for (int r = 0; r < CS; ++r) *(volatile int*)cluster.map_shared_rank(&s_abort, r) = 1;
        }
      }
    };
    // (the block-flat loop measured slower here: per-row fixed costs dominate, keep the VW loop)
    products<false, true, int, 1024>(false, a.a_rpt, a.a_col, nullptr, a.b_rpt, a.b_col, nullptr, row,
                                     rank * 1024 + t, CS * 1024, a.vw_log2, f, stop, a.long_len, &s_lcnt);
    if (a.long_len > 0) {
      // the deferred rows of any CTA are split over all CTAs: every CTA must run the pass
      __syncthreads();
      if (t == 0) s_lcnt = 1;
      for_long_products<false, true, int>(a.a_rpt, a.a_col, nullptr, a.b_rpt, a.b_col, nullptr, true, row, t, 1024,
                                          a.long_len, s_list, &s_lcnt, &s_bf, f, stop, rank, CS);
    }
    (void)mine;
    cluster.sync();
    if (rank == 0 && t == 0) {
      if (s_abort) {
        overflow2[atomicAdd(count2, 1)] = row;  // recount in global memory
      } else {
        a.c_cnt[row] = s_cnt;
      }
    }
    cluster.sync();
  }
}

template <typename VT, int CS>
__global__ void __launch_bounds__(1024) k_num_cluster(NumArgs a) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  constexpr int Ts = kClusterNumSlots;
  __shared__ int* s_kp[CS];
  __shared__ VT* s_vp[CS];
  __shared__ int s_list[kLongChunk], s_lcnt;
  __shared__ BlockFlat<VT> s_bf;
  __shared__ int s_lohi[2];
  __shared__ long long s_part[CS];
  __shared__ long long ws[33];
  cg::cluster_group cluster = cg::this_cluster();
  const int rank = (int)cluster.block_rank();
  const int t = threadIdx.x;
  VT* Vloc = reinterpret_cast<VT*>(smem_raw);
  int* Kloc = reinterpret_cast<int*>(Vloc + Ts);
  if (t < CS) {
    s_kp[t] = cluster.map_shared_rank(Kloc, t);
    s_vp[t] = cluster.map_shared_rank(Vloc, t);
  }
  int* lohi0 = cluster.map_shared_rank(s_lohi, 0);
  const long long nclusters = gridDim.x / CS;
  const long long cid = blockIdx.x / CS;
  unsigned* bits = reinterpret_cast<unsigned*>(static_cast<unsigned char*>(a.slab) + cid * a.slab_stride);
  unsigned* pre = bits + a.bitmap_words;
  const CKeys K{s_kp, 31 - __clz(Ts), Ts - 1};
  const CVals<VT> V{s_vp, 31 - __clz(Ts), Ts - 1};
  const unsigned mask = CS * Ts - 1;
  // rows are handed out dynamically (one global counter per launch; rank 0 fetches, the cluster
  // reads it through DSMEM): row costs vary by 10x within a group (measured 3x span/mean imbalance
  // with the static cid-strided assignment)
  __shared__ long long s_next;
  const long long* next0 = cluster.map_shared_rank(&s_next, 0);
  (void)nclusters; (void)cid;
  while (true) {
    if (rank == 0 && t == 0) s_next = a.row_counter ? (long long)atomicAdd(a.row_counter, 1) : 0;
    cluster.sync();
    const long long i = *(volatile const long long*)next0;
    cluster.sync();  // every CTA has read it: rank 0 may overwrite it or exit
    if (i >= a.nrows) break;  // cluster-uniform
    const int row = a.rows[i];
    if (a.prof && rank == 0 && t == 0) a.prof[4 * i + 1] = gtimer();
    int4* k4 = reinterpret_cast<int4*>(Kloc);
    for (int s = t; s < Ts / 4; s += 1024) k4[s] = make_int4(-1, -1, -1, -1);
    for (int s = t; s < Ts; s += 1024) Vloc[s] = VT(0);
    if (t == 0) { s_lcnt = 0; s_lohi[0] = INT_MAX; s_lohi[1] = -1; }
    cluster.sync();
    // (a) accumulate over the distributed table
    auto f = [&](int key, VT prod) {
      bool ins;
      const unsigned s = probe(K, mask, key, ins);
      V.add(s, prod);
    };
    products<true, false, VT, 1024>(false, a.a_rpt, a.a_col, static_cast<const VT*>(a.a_val), a.b_rpt, a.b_col,
                                    static_cast<const VT*>(a.b_val), row, rank * 1024 + t, CS * 1024, a.vw_log2,
                                    f, NoStop{}, a.long_len, &s_lcnt);
    if (a.long_len > 0) {
      // the deferred rows of any CTA are split over all CTAs: every CTA must run the pass
      __syncthreads();
      if (t == 0) s_lcnt = 1;
      for_long_products<true, false, VT>(a.a_rpt, a.a_col, static_cast<const VT*>(a.a_val), a.b_rpt, a.b_col,
                                         static_cast<const VT*>(a.b_val), true, row, t, 1024, a.long_len, s_list,
                                         &s_lcnt, &s_bf, f, NoStop{}, rank, CS);
    }
    cluster.sync();
    if (a.prof && rank == 0 && t == 0) a.prof[4 * i + 2] = gtimer();
    // (b) column span of the row: min/max over every slice, reduced into CTA 0
    {
      int mn = INT_MAX, mx = -1;
      for (int s = t; s < Ts; s += 1024) {
        const int k = Kloc[s];
        if (k >= 0) { mn = min(mn, k); mx = max(mx, k); }
      }
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) {
        mn = min(mn, __shfl_xor_sync(0xffffffffu, mn, o));
        mx = max(mx, __shfl_xor_sync(0xffffffffu, mx, o));
      }
      if ((t & 31) == 0 && mx >= 0) { atomicMin(lohi0, mn); atomicMax(lohi0 + 1, mx); }
    }
    cluster.sync();
    const int lo = lohi0[0], hi = lohi0[1];
    const int W = hi >= lo ? (int)(((unsigned)(hi - lo)) >> 5) + 1 : 0;
    const int wper = (W + CS - 1) / CS;
    const int wa = min(W, rank * wper), wb = min(W, wa + wper);
    for (int w = wa + t; w < wb; w += 1024) bits[w] = 0u;
    cluster.sync();
    // (c) bitmap over [lo, hi] in global scratch, prefix popcounts, rank, write C
    for (int s = t; s < Ts; s += 1024) {
      const int k = Kloc[s];
      if (k >= 0) atomicOr(bits + ((k - lo) >> 5), 1u << ((k - lo) & 31));
    }
    cluster.sync();
    {
      // prefix popcounts over this CTA's word slice [wa, wb): warp-contiguous segments read
      // lane-interleaved (coalesced), warp scans per 32 words
      const int lane = t & 31, wid = t >> 5;
      const int seg = (((wb - wa) + 1023) / 1024) * 32;  // words per warp, multiple of 32
      const int s0 = wa + wid * seg, s1 = min(wb, s0 + seg);
      unsigned loc = 0;
      for (int w = s0 + lane; w < s1; w += 32) loc += __popc(bits[w]);
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) loc += __shfl_xor_sync(0xffffffffu, loc, o);
      long long tot;
      long long run = Grp<1024>::excl_scan(lane == 0 ? (long long)loc : 0LL, &tot, ws);
      run = __shfl_sync(0xffffffffu, run, 0);
      if (t == 0) {
        for (int r = 0; r < CS; ++r) cluster.map_shared_rank(s_part, r)[rank] = tot;
      }
      cluster.sync();
      for (int r = 0; r < rank; ++r) run += s_part[r];
      for (int w0 = s0; w0 < s1; w0 += 32) {
        const int w = w0 + lane;
        const unsigned v = w < s1 ? __popc(bits[w]) : 0u;
        unsigned incl = v;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
          const unsigned y = __shfl_up_sync(0xffffffffu, incl, o);
          if (lane >= o) incl += y;
        }
        if (w < s1) pre[w] = (unsigned)(run + incl - v);
        run += __shfl_sync(0xffffffffu, incl, 31);
      }
    }
    cluster.sync();
    const long long c0 = a.c_rpt[row];
    const long long cn = a.c_rpt[row + 1] - c0;
    if (rank == 0 && t == 0) {
      long long total = 0;
      for (int r = 0; r < CS; ++r) total += s_part[r];
      if (total != cn) atomicOr(a.err_flags, 2);
    }
    VT* __restrict__ cv = static_cast<VT*>(a.c_val) + c0;
    int32_t* __restrict__ cc = a.c_col + c0;
    for (int s = t; s < Ts; s += 1024) {
      const int k = Kloc[s];
      if (k < 0) continue;
      const unsigned d = (unsigned)(k - lo);
      const long long r = (long long)pre[d >> 5] + __popc(bits[d >> 5] & ((1u << (d & 31)) - 1u));
      if (r < cn) { cc[r] = k; cv[r] = Vloc[s]; }
    }
    cluster.sync();
    if (a.prof && rank == 0 && t == 0) {
      unsigned smid;
      asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
      a.prof[4 * i + 3] = gtimer();
      a.prof[4 * i + 0] = ((unsigned long long)smid << 32) | (unsigned)row;
    }
  }
}

template <typename K>
cudaError_t set_cluster_attrs(K kernel, int smem) {
  cudaError_t e = cudaFuncSetAttribute(kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  if (e == cudaSuccess) e = cudaFuncSetAttribute(kernel, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
  return e;
}

template <typename K, typename... Args>
cudaError_t launch_cluster(cudaStream_t s, K kernel, int cs, int nclusters, int smem, Args... args) {
  cudaLaunchConfig_t cfg{};
  cfg.gridDim = dim3((unsigned)(nclusters * cs));
  cfg.blockDim = dim3(1024);
  cfg.dynamicSmemBytes = (size_t)smem;
  cfg.stream = s;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeClusterDimension;
  attr[0].val.clusterDim.x = cs;
  attr[0].val.clusterDim.y = 1;
  attr[0].val.clusterDim.z = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  return cudaLaunchKernelEx(&cfg, kernel, args...);
}

template <typename K>
int max_clusters(K kernel, int cs, int smem) {
  cudaLaunchConfig_t cfg{};
  cfg.gridDim = dim3(cs);
  cfg.blockDim = dim3(1024);
  cfg.dynamicSmemBytes = (size_t)smem;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeClusterDimension;
  attr[0].val.clusterDim.x = cs;
  attr[0].val.clusterDim.y = 1;
  attr[0].val.clusterDim.z = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  int n = 0;
  if (cudaOccupancyMaxActiveClusters(&n, kernel, &cfg) != cudaSuccess) {
    cudaGetLastError();
    n = 0;
  }
  return n > 0 ? n : 1;
}

}  // namespace

int cluster_capacity_sym() { return kClusterSize * kClusterSymSlots; }
int cluster_capacity_num() { return kClusterSize * kClusterNumSlots; }

cudaError_t launch_symbolic_cluster(cudaStream_t s, const SymArgs& a, const int32_t* rows, const int* count,
                                    int32_t* overflow2, int* count2, int fill_limit, int max_rows) {
  if (max_rows <= 0) return cudaSuccess;
  constexpr int smem = kClusterSymSlots * 4;
  static PerDevice ncache;
  auto& ncd = ncache.here();
  if (ncd.load() == 0) {
    cudaError_t e = set_cluster_attrs(k_sym_cluster<kClusterSize>, smem);
    if (e != cudaSuccess) return e;
    ncd.store(max_clusters(k_sym_cluster<kClusterSize>, kClusterSize, smem));
  }
  const int nc = (int)ncd.load();
  SymArgs b = a;
  if (b.vw_log2 > 5) b.vw_log2 = 5;
  const int grid = max_rows < nc ? max_rows : nc;
  return launch_cluster(s, k_sym_cluster<kClusterSize>, kClusterSize, grid, smem, b, rows, count, overflow2, count2,
                        fill_limit);
}

template <typename VT, int CS>
cudaError_t launch_num_cluster_cs(cudaStream_t s, const NumArgs& a, int* nclusters_out) {
  constexpr int smem = kClusterNumSlots * ((int)sizeof(VT) + 4);
  static PerDevice ncache;
  auto& ncd = ncache.here();
  if (ncd.load() == 0) {
    cudaError_t e = set_cluster_attrs(k_num_cluster<VT, CS>, smem);
    if (e != cudaSuccess) return e;
    ncd.store(max_clusters(k_num_cluster<VT, CS>, CS, smem));
  }
  const int nc = (int)ncd.load();
  if (nclusters_out) { *nclusters_out = nc; return cudaSuccess; }  // query only
  if (a.nrows <= 0) return cudaSuccess;
  NumArgs b = a;
  if (b.vw_log2 > 5) b.vw_log2 = 5;
  const int grid = (int)(a.nrows < nc ? a.nrows : nc);
  return launch_cluster(s, k_num_cluster<VT, CS>, CS, grid, smem, b);
}

cudaError_t launch_numeric_cluster(cudaStream_t s, bool fp64, int cs, const NumArgs& a, int* nclusters_out) {
  switch (cs) {
    case 2: return fp64 ? launch_num_cluster_cs<double, 2>(s, a, nclusters_out) : launch_num_cluster_cs<float, 2>(s, a, nclusters_out);
    case 4: return fp64 ? launch_num_cluster_cs<double, 4>(s, a, nclusters_out) : launch_num_cluster_cs<float, 4>(s, a, nclusters_out);
    case 8: return fp64 ? launch_num_cluster_cs<double, 8>(s, a, nclusters_out) : launch_num_cluster_cs<float, 8>(s, a, nclusters_out);
    default: return cudaErrorInvalidValue;
  }
}

}  // namespace spg
