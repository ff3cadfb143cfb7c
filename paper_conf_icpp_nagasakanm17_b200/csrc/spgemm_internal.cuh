// spgemm_internal.cuh — group tables, device primitives and launcher declarations shared by
// the kernels of libspgemm.so (B200 / sm_100a).  Nothing here is shared with oracle/.
//
// Paper map (PAPER.md line numbers):
//   Alg. 2 n_prod count ........ :90-96   -> k_nprod_group       (kernels_setup.cu)
//   grouping (2)/(6) ........... :84-88   -> k_group_scatter     (kernels_setup.cu)
//   Alg. 3/4 thread assignment . :102-126 -> for_each_product    (sub-groups of VW lanes)
//   Alg. 5 hash insert ......... :130-153 -> probe<SKeys|GKeys> (below)
//   group-0 overflow retry ..... :155,181 -> optimistic group + k_sym_global
//   calculation + gather + sort  :171-173 -> num_row (bucket-rank sort)
//   Table I / parameter rule ... :157-183 -> kSymGroups / kNumGroups (B200 values)
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

#include <atomic>
#include <climits>

namespace spg {

constexpr unsigned kHashScal = 107u;  // HASH_SCAL; any odd constant (reading R4)
// Reading R4: the slot is the TOP log2(t_size) bits of key * 2654435761 mod 2^32
// (Knuth's multiplicative hash) instead of (key * HASH_SCAL) mod t_size.  The low bits of key * odd
// depend only on the key's low bits, which are biased on R-MAT columns (bit = 1 with p = 0.4):
// R-MAT s22 symbolic 19.0 -> 16.0 ms, QCD-like numeric 0.65 -> 0.53 ms, FEM shapes unchanged.
// SPG_HASH_FIB 0 restores the paper's low-bits form (ablation builds).
#ifndef SPG_HASH_FIB
#define SPG_HASH_FIB 1
#endif
constexpr int kMaxGroups = 24;
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
// Threads per row target ~8-16 products per thread at the group's bound (per-warp fixed costs
// dominate below that).
constexpr GroupSpec kSymGroups[] = {
    {16, 32, 4, 256},        {32, 64, 8, 256},         {128, 256, 16, 256},
    {256, 512, 32, 256},     {512, 1024, 32, 256},     {1024, 2048, 64, 64},
    {2048, 4096, 128, 128},  {4096, 8192, 256, 256},   {8192, 16384, 512, 512},
    {16384, 32768, 1024, 1024},
    {-1, 32768, 1024, 1024},  // optimistic (no upper bound)
};
constexpr int kNumSymBounds = 10;   // groups 0..9 have an upper bound
constexpr int kSymOptimistic = 10;
constexpr int kSymGlobal = 11;
constexpr int kSymRange = 12;       // range rows: warp-per-row offset table (kernels_range.cu)
constexpr int kNumSymGroups = 13;   // including global and range

// Phase 2 (numeric), key = nnz_i.  Same bounds for fp32 and fp64 (fp64 sizes the smem).
// Groups 10-12 = cluster-per-row (DSMEM of 2/4/8 CTAs, kernels_cluster.cu; load factor up to 3/4
// so an 8-CTA cluster covers the heaviest rows of the graph configs), 13 = global.
constexpr int kClusterSize = 8;
constexpr int kClusterSymSlots = 32768;  // int keys per CTA (128 KB)
constexpr int kClusterNumSlots = 16384;  // key+value slots per CTA (128 KB fp32, 192 KB fp64)
constexpr GroupSpec kNumGroups[] = {
    {8, 16, 4, 256},         {16, 32, 8, 256},         {64, 128, 16, 256},
    {128, 256, 32, 256},     {256, 512, 64, 64},       {512, 1024, 128, 128},
    {1024, 2048, 256, 256},  {2048, 4096, 512, 512},   {4096, 8192, 1024, 1024},
    {8192, 16384, 1024, 1024},
    {2 * kClusterNumSlots * 3 / 4, 2 * kClusterNumSlots, 2 * 1024, 1024},   // cluster of 2 CTAs
    {4 * kClusterNumSlots * 3 / 4, 4 * kClusterNumSlots, 4 * 1024, 1024},   // cluster of 4 CTAs
    {8 * kClusterNumSlots * 3 / 4, 8 * kClusterNumSlots, 8 * 1024, 1024},   // cluster of 8 CTAs
};
constexpr int kNumNumBounds = 13;
constexpr int kNumCluster = 10;  // groups 10, 11, 12: clusters of 2, 4, 8 CTAs
constexpr int kNumGlobal = 13;
constexpr int kNumRange = 14;       // range rows (kernels_range.cu)
// Batched expand-bucket-rank rows (kernels_esc.cu): numeric groups 15..20 hold the rows of
// symbolic groups 2..7 whose n_prod_i <= ESC_PCT/100 * nnz_i (weak compression); a batch of them
// fits one CTA because the symbolic group bounds n_prod_i.
constexpr int kNumEscBase = 15;
constexpr int kEscSymLo = 2, kEscSymHi = 7;
constexpr int kNumNumGroups = kNumEscBase + (kEscSymHi - kEscSymLo + 1);  // 21

// Range rows (kernels_range.cu): column span R_i <= kRangeMaxSpan and
// R_i <= kRangeSpanPerProd * n_prod_i, n_prod_i in [range_min_np, kRangeMaxNprod] (one warp
// per row).  Per-CTA shared-memory budget of the per-warp tables (the rest of the SM's 256 KB
// stays L1 for the B rows the CTA's neighbouring rows share).
constexpr int kRangeMaxSpan = 2048;
constexpr int kRangeSpanPerProd = 4;
constexpr long long kRangeMaxNprod = 1 << 16;
constexpr long long kRangeMinNprodDefault = 256;
constexpr long long kRangeSmemBudget = 96 * 1024;

// Numeric per-row shared-memory layout: vals[T] | keys[T] | bucket[NB+1] | sidx[upper] ,
// NB = T/2 (T/8 for the largest table) buckets for the bucket-rank sort.
__host__ __device__ constexpr int num_nbuckets(int T) { return T <= 8192 ? T / 2 : T / 8; }
__host__ __device__ constexpr int align16(int x) { return (x + 15) & ~15; }
template <typename VT>
__host__ __device__ constexpr int num_row_bytes(int T, long long upper) {
  return align16(T * (int)sizeof(VT) + T * 4 + (num_nbuckets(T) + 1) * 4 + (int)upper * 2 + 8);
}
// CTA-per-row numeric groups with the two-level bitmap rank (kernels_numeric.cu):
// vals[T] | keys[T] | fine[upper] u32 | pre2[upper] u16 | lvl1[l1] u32 | pre1[l1] u32
template <typename VT>
__host__ __device__ constexpr long long num_cta_bytes(int T, long long upper, long long l1) {
  return align16(T * (int)sizeof(VT) + T * 4 + (int)upper * 6) + l1 * 8 + 16;
}

// ----------------------------------------------------------------------------- per-device setup
// One-time per-kernel settings (dynamic shared memory opt-in, cluster occupancy) belong to the
// device context, so launchers keep them per device ordinal; atomics make concurrent first
// launches from several host threads safe (a setting applied twice is harmless).
constexpr int kMaxDevices = 64;
struct PerDevice {
  std::atomic<long long> v[kMaxDevices] = {};
  std::atomic<long long>& here() {
    int d = 0;
    if (cudaGetDevice(&d) != cudaSuccess || d < 0) d = 0;
    return v[d % kMaxDevices];
  }
};

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
  int overflow2_count;  // rows that overflowed the cluster table too (-> global memory)
  int err_flags;  // bit0 invalid input, bit1 numeric row count mismatch
  int b_unsorted;  // some B row is not strictly increasing (disables private accumulators)
  int cursor[2][kMaxGroups];
  int range_rmax;  // max column span R_i over the range rows (sizes the per-warp tables)
  int row_counter[4];  // numeric cluster groups: dynamic row counters (zeroed per numeric call)
  int defer_count[2];  // step (1): deferred long rows of B (0) and A (1)
  int bbits_wmax;      // range rows: max words of a B-row bitmap (k_brow_bits)
  int small_overflow;  // small-matrix path: rows with n_prod_i > kSmallCap (-> general path)
  long long ends[4];   // small-matrix path: a_rpt[0], a_rpt[m], b_rpt[0], b_rpt[k]
};

// Small matrices (m <= kSmallRows): one-launch symbolic and numeric phases, thread per row with a
// register table of kSmallCap slots (kernels_tiny.cu), no grouping and no sync 1.
constexpr long long kSmallRows = 65536;
constexpr int kSmallCap = 32;

struct Bounds {  // group bounds passed by value
  long long upper[kMaxGroups];
  int nbounds;     // groups 0..nbounds-1 bounded; key > last bound -> group nbounds
  int min_group;   // -1 or forced minimum group
  int range_group;  // -1, or the group id of range rows (kSymRange / kNumRange)
  long long range_min_np;  // phase 1: n_prod lower bound of range rows
  long long range_k;       // phase 1: rows of B (range rows need rpt_B[k] < 2^31: 32-bit offsets)
};

struct Offsets {
  long long off[kMaxGroups + 1];
  int ngroups;
};

// ----------------------------------------------------------------------------- primitives
__device__ __forceinline__ int ld_volatile(const int* p) { return *(const volatile int*)p; }

// Explicit shared-memory access through 32-bit shared-window addresses (keeps the
// generic->shared conversion out of the hot loops).  No "memory" clobbers: global loads may
// be scheduled across them; the volatile asm statements keep their mutual order.
// opaque(): hide a loop-invariant value's derivation so ptxas keeps it in a register instead of
// rematerialising it (S2R SR_CgaCtaId for shared windows; 64-bit re-association for pointers).
__device__ __forceinline__ unsigned opaque(unsigned x) { asm volatile("" : "+r"(x)); return x; }
template <typename T>
__device__ __forceinline__ T* opaque(T* p) { asm volatile("" : "+l"(p)); return p; }
__device__ __forceinline__ unsigned smem_u32(const void* p) { return opaque((unsigned)__cvta_generic_to_shared(p)); }
__device__ __forceinline__ int lds_s32(unsigned a) {
  int v;
  asm volatile("ld.shared.b32 %0, [%1];" : "=r"(v) : "r"(a));
  return v;
}
__device__ __forceinline__ int cas_s32(unsigned a, int cmp, int val) {
  int old;
  asm volatile("atom.shared.cas.b32 %0, [%1], %2, %3;" : "=r"(old) : "r"(a), "r"(cmp), "r"(val));
  return old;
}
__device__ __forceinline__ void st_s8(unsigned a, int v) { asm volatile("st.shared.u8 [%0], %1;" ::"r"(a), "r"(v)); }
__device__ __forceinline__ void red_or_s(unsigned a, unsigned v) { asm volatile("red.shared.or.b32 [%0], %1;" ::"r"(a), "r"(v)); }
__device__ __forceinline__ void red_add_s(unsigned a, float v) { asm volatile("red.shared.add.f32 [%0], %1;" ::"r"(a), "f"(v)); }
__device__ __forceinline__ void red_add_s(unsigned a, double v) { asm volatile("red.shared.add.f64 [%0], %1;" ::"r"(a), "d"(v)); }

// Key tables in shared (SKeys) or global (GKeys) memory with one probe interface.
struct SKeys {
  unsigned base;  // shared address of slot 0
  __device__ __forceinline__ int ld(unsigned h) const { return lds_s32(base + 4u * h); }
  __device__ __forceinline__ int cas(unsigned h, int c, int v) const { return cas_s32(base + 4u * h, c, v); }
};
struct GKeys {
  int* p;
  // ld.global.cg (L2, not L1-cached, not volatile): a slot changes only once (-1 -> key), so a
  // stale -1 merely makes the following CAS report the real key; probes of independent
  // products may overlap.
  __device__ __forceinline__ int ld(unsigned h) const { return __ldcg(p + h); }
  __device__ __forceinline__ int cas(unsigned h, int c, int v) const { return atomicCAS(p + h, c, v); }
};
template <typename VT>
struct SVals {
  unsigned base;
  __device__ __forceinline__ void add(unsigned h, VT v) const { red_add_s(base + (unsigned)sizeof(VT) * h, v); }
};
template <typename VT>
struct GVals {
  VT* p;
  __device__ __forceinline__ void add(unsigned h, VT v) const { atomicAdd(p + h, v); }
};

// Algorithm 5 on either table kind: key = col_B[k]; hash = the multiplicative
// hash of key into t_size slots (t_size a power of two; its top bits, reading R4
// above); linear probing; empty slot = -1;
// insert by atomicCAS.  Returns the slot of `key`; inserted = this call added it (nz++).
template <typename Keys>
__device__ __forceinline__ unsigned probe(const Keys& K, unsigned mask, int key, bool& inserted) {
#if SPG_HASH_FIB
  unsigned h = ((unsigned)key * 2654435761u) >> __clz(mask);
#else
  unsigned h = ((unsigned)key * kHashScal) & mask;
#endif
  inserted = false;
  while (true) {
    const int cur = K.ld(h);
    if (cur == key) return h;
    if (cur == -1) {
      const int old = K.cas(h, -1, key);
      if (old == -1) { inserted = true; return h; }
      if (old == key) return h;
    }
    h = (h + 1) & mask;
  }
}

// Iterate the intermediate products of one row (Alg. 3/4 loops generalised): sub-groups of
// VW lanes walk the row's A non-zeros, lanes stride VW over each B row.  Two-stage software
// pipeline over A non-zeros: while B row j is processed, rpt_B of j+1 and col_A of j+2 are
// already in flight; B rows are unrolled by 2 so each lane has two gathers outstanding.
// f(key, value) is called per product; stop() (checked per product when CHECK_STOP) aborts.
// Load balance (CTA-per-row groups): with long_len > 0 a sub-group skips B rows longer than
// long_len; the caller then runs for_long_products, where the whole CTA walks each of them
// (hub columns of power-law graphs would otherwise serialise a CTA behind one sub-group).
template <bool NUM, bool CHECK_STOP, typename VT, bool WSYNC = false, typename F, typename S>
__device__ __forceinline__ void for_each_product(const int64_t* __restrict__ a_rpt, const int32_t* __restrict__ a_col,
                                                 const VT* __restrict__ a_val, const int64_t* __restrict__ b_rpt,
                                                 const int32_t* __restrict__ b_col, const VT* __restrict__ b_val,
                                                 int row, int t, int tpr, int vwl, F&& f, S&& stop,
                                                 int long_len = 0, int* deferred = nullptr) {
  const long long a0 = __ldg(a_rpt + row);
  const int na = (int)(__ldg(a_rpt + row + 1) - a0);  // row-relative 32-bit indexing
  const int32_t* __restrict__ ac = opaque(a_col + a0);
  const VT* __restrict__ avp = NUM ? opaque(a_val + a0) : nullptr;
  const int vw = 1 << vwl, sub = t >> vwl, lane = t & (vw - 1), nsub = tpr >> vwl;
  // WSYNC: reconverge the sub-group after every A non-zero (callers that update per-sub-group
  // private accumulators with plain read-modify-writes rely on it)
  const unsigned sg = vw >= 32 ? 0xffffffffu : (((1u << vw) - 1u) << ((threadIdx.x & 31) & ~(vw - 1)));
  // Sub-group `sub` owns A non-zeros sub, sub + nsub, sub + 2*nsub, ... (Alg. 4's warp-per-a_ik,
  // interleaved); they are taken in batches of vw: lane l fetches the metadata of the l-th
  // non-zero of the batch (col_A, val_A, rpt_B pair — vw independent gathers in flight, the next
  // batch prefetched), then the sub-group walks the batch with shuffle broadcasts.
  const int stride = nsub * vw;
  int jb = sub + nsub * lane;  // this lane's non-zero in the current batch
  if (sub >= na) return;
  int kk = 0, len = 0;
  long long b0 = 0;
  VT av = VT(0);
  if (jb < na) {
    kk = __ldg(ac + jb);
    if (NUM) av = __ldg(avp + jb);
    b0 = __ldg(b_rpt + kk);
    len = (int)(__ldg(b_rpt + kk + 1) - b0);
  }
  for (int base = sub; base < na; base += stride) {
    const int cnt = min(vw, (na - base + nsub - 1) / nsub);  // sub-group-uniform
    // prefetch the next batch
    const int jn = jb + stride;
    int kkn = 0, lenn = 0;
    long long b0n = 0;
    VT avn = VT(0);
    if (jn < na) {
      kkn = __ldg(ac + jn);
      if (NUM) avn = __ldg(avp + jn);
      b0n = __ldg(b_rpt + kkn);
      lenn = (int)(__ldg(b_rpt + kkn + 1) - b0n);
    }
    for (int e = 0; e < cnt; ++e) {
      const long long eb0 = __shfl_sync(sg, b0, e, vw);
      int elen = __shfl_sync(sg, len, e, vw);
      const VT eav = NUM ? __shfl_sync(sg, av, e, vw) : VT(0);
      if (long_len > 0 && elen > long_len) {  // deferred to for_long_products
        elen = 0;
        if (deferred) *deferred = 1;
      }
      const int32_t* __restrict__ bc = opaque(b_col + eb0);
      const VT* __restrict__ bv = NUM ? opaque(b_val + eb0) : nullptr;
#pragma unroll 1
      for (int q = lane; q < elen; q += 2 * vw) {
        const int k0 = __ldg(bc + q);
        const VT v0 = NUM ? __ldg(bv + q) : VT(0);
        const bool h1 = q + vw < elen;
        int k1 = 0;
        VT v1 = VT(0);
        if (h1) { k1 = __ldg(bc + q + vw); if (NUM) v1 = __ldg(bv + q + vw); }
        // CHECK_STOP: a stopped lane skips its products (at most one insert after the flag is
        // raised); the sub-group leaves together at the next entry boundary.
        if (!(CHECK_STOP && stop())) f(k0, eav * v0);
        if (h1 && !(CHECK_STOP && stop())) f(k1, eav * v1);
      }
      if constexpr (WSYNC || CHECK_STOP) __syncwarp(sg);
      if constexpr (CHECK_STOP) {
        if (__any_sync(sg, stop())) return;
      }
    }
    jb = jn; kk = kkn; av = avn; b0 = b0n; len = lenn;
  }
}

// Load-balanced variant for short B rows (graphs): groups of G lanes (G = min(TPR, 32)) take
// batches of G consecutive A non-zeros, scan their B-row lengths, and lane l handles products
// l, l+G, l+2G, ... of the concatenated batch, finding its A non-zero by a log2(G)-step shuffle
// binary search — every lane does the same work whatever the B-row lengths (the VW-per-entry
// loop leaves most lanes idle on 2-4-entry rows and serialises on 30-60-entry rows).
template <bool NUM, bool CHECK_STOP, typename VT, int G, typename F, typename S>
__device__ __forceinline__ void for_each_product_flat(const int64_t* __restrict__ a_rpt,
                                                      const int32_t* __restrict__ a_col,
                                                      const VT* __restrict__ a_val,
                                                      const int64_t* __restrict__ b_rpt,
                                                      const int32_t* __restrict__ b_col,
                                                      const VT* __restrict__ b_val, int row, int t, int tpr,
                                                      F&& f, S&& stop, int long_len, int* deferred) {
  const long long a0 = __ldg(a_rpt + row);
  const int na = (int)(__ldg(a_rpt + row + 1) - a0);
  const int32_t* __restrict__ ac = opaque(a_col + a0);
  const VT* __restrict__ avp = NUM ? opaque(a_val + a0) : nullptr;
  const int gl = t % G, gi = t / G, ng = tpr / G;
  const unsigned gm = G >= 32 ? 0xffffffffu : (((1u << G) - 1u) << ((threadIdx.x & 31) & ~(G - 1)));
  for (int base = gi * G; base < na; base += ng * G) {  // uniform within the group
    const int j = base + gl;
    int len = 0;
    long long b0 = 0;
    VT av = VT(0);
    if (j < na) {
      const int kk = __ldg(ac + j);
      if (NUM) av = __ldg(avp + j);
      b0 = __ldg(b_rpt + kk);
      len = (int)(__ldg(b_rpt + kk + 1) - b0);
      if (long_len > 0 && len > long_len) {  // deferred to for_long_products
        len = 0;
        if (deferred) *deferred = 1;
      }
    }
    int incl = len;
#pragma unroll
    for (int d = 1; d < G; d <<= 1) {
      const int y = __shfl_up_sync(gm, incl, d, G);
      if (gl >= d) incl += y;
    }
    const int total = __shfl_sync(gm, incl, G - 1, G);
    // kFlatU products per lane per round: all their gathers are issued before the first table
    // update (the B rows of graph shapes are short and scattered: each gather is an L2/HBM trip)
    constexpr int kFlatU = 4;
    for (int p0 = 0; p0 < total; p0 += G * kFlatU) {
      int keys[kFlatU];
      VT vals[kFlatU];
#pragma unroll
      for (int u = 0; u < kFlatU; ++u) {
        const int p = p0 + u * G + gl;
        int e = 0;
#pragma unroll
        for (int st = G / 2; st > 0; st >>= 1)
          if (__shfl_sync(gm, incl, e + st - 1, G) <= p) e += st;
        const int ie = __shfl_sync(gm, incl, e, G);
        const int le = __shfl_sync(gm, len, e, G);
        const long long be = __shfl_sync(gm, b0, e, G);
        const VT ae = NUM ? __shfl_sync(gm, av, e, G) : VT(0);
        keys[u] = -1;
        if (p < total) {
          const long long q = be + (p - (ie - le));
          keys[u] = __ldg(b_col + q);
          if (NUM) vals[u] = ae * __ldg(b_val + q);
        }
      }
#pragma unroll
      for (int u = 0; u < kFlatU; ++u)
        if (keys[u] >= 0 && !(CHECK_STOP && stop())) f(keys[u], NUM ? vals[u] : VT(0));
    }
    if constexpr (CHECK_STOP) {
      if (__any_sync(gm, stop())) return;
    }
  }
}

// CTA-level flattened loop for CTA-per-row groups (every thread of the CTA must call it): the
// row's A non-zeros are taken in chunks of kFlatChunk; their metadata and the inclusive scan of
// their B-row lengths go to shared memory (BlockFlat), and all tpr threads stride the chunk's
// concatenated products, each locating its A non-zero by binary search over the scan.  Equal
// work per thread whatever the B-row lengths — no long-row deferral needed.
constexpr int kFlatChunk = 256;
template <int TPR>
struct Grp;  // row-group collectives (defined below)
// N entries per chunk: kFlatChunk by default; the CTA-per-row group kernels use one chunk of TPR
// entries (up to 1024) so that a row of <= TPR A non-zeros costs a single metadata round trip.
// NB > 0: a block-start table — for each 32-product block of the chunk, the first A entry holding
// one of its products — so a product finds its entry with one lookup and a short forward walk
// instead of a binary search over the chunk (chunks of up to 32 * NB products; larger ones search).
template <typename VT, int N = kFlatChunk, int NB = 0>
struct BlockFlat {
  static constexpr int kN = N;
  static constexpr int kNB = NB;
  long long b0[N];
  int incl[N];
  VT av[N];
  int bstart[NB > 0 ? NB : 1];
};
template <int TPR>
constexpr int flat_chunk_of() { return TPR < 1024 ? TPR : 1024; }
template <bool NUM, bool CHECK_STOP, typename VT, int TPR, typename BF, typename F, typename S>
__device__ __forceinline__ void for_each_product_block(const int64_t* __restrict__ a_rpt,
                                                       const int32_t* __restrict__ a_col,
                                                       const VT* __restrict__ a_val,
                                                       const int64_t* __restrict__ b_rpt,
                                                       const int32_t* __restrict__ b_col,
                                                       const VT* __restrict__ b_val, bool active, int row, int t,
                                                       BF* sh, long long* ws, F&& f, S&& stop,
                                                       int part = 0, int nparts = 1) {
  static_assert(TPR > 32, "CTA-level loop");
  constexpr int CH = TPR < BF::kN ? TPR : BF::kN;
  constexpr int tpr = TPR;
  const long long a0 = active ? __ldg(a_rpt + row) : 0;
  const int na = active ? (int)(__ldg(a_rpt + row + 1) - a0) : 0;  // CTA-uniform
  const int32_t* __restrict__ ac = a_col + a0;
  for (int c = part * CH; c < na; c += nparts * CH) {
    const int cn = min(CH, na - c);
    int len = 0;
    if (t < cn) {
      const int kk = __ldg(ac + c + t);
      const long long b0 = __ldg(b_rpt + kk);
      len = (int)(__ldg(b_rpt + kk + 1) - b0);
      sh->b0[t] = b0;
      if (NUM) sh->av[t] = __ldg(a_val + a0 + c + t);
    }
    long long tot;
    const long long ex = Grp<TPR>::excl_scan(t < cn ? len : 0, &tot, ws);  // block scan
    if (t < cn) sh->incl[t] = (int)(ex + len);
    const int P = (int)tot;  // CTA-uniform
    const bool table = BF::kNB > 0 && P <= 32 * BF::kNB;
    if (table && t < cn)  // 32-product blocks whose first product lies in this entry
      for (int k = (int)((ex + 31) >> 5); k < (int)((ex + len + 31) >> 5); ++k) sh->bstart[k] = t;
    __syncthreads();
    // kU products per thread per round: all kU gathers are issued before any table update (B rows
    // of graph shapes are short and scattered: each gather is an L2/HBM round trip)
    constexpr int kU = 4;
#pragma unroll 1
    for (int p0 = t; p0 < P; p0 += kU * tpr) {
      int keys[kU];
      VT vals[kU];
      int es[kU];
#pragma unroll
      for (int u = 0; u < kU; ++u) {
        const int p = p0 + u * tpr;
        es[u] = -1;
        if (p < P) {
          int lo;  // first e with incl[e] > p
          if (table) {
            lo = sh->bstart[p >> 5];
            while (sh->incl[lo] <= p) ++lo;
          } else {
            lo = 0;
            int hi = cn - 1;
            while (lo < hi) {
              const int mid = (lo + hi) >> 1;
              if (sh->incl[mid] <= p) lo = mid + 1; else hi = mid;
            }
          }
          es[u] = lo;
          const int start = lo ? sh->incl[lo - 1] : 0;
          const long long q = sh->b0[lo] + (p - start);
          keys[u] = __ldg(b_col + q);
          vals[u] = NUM ? __ldg(b_val + q) : VT(0);
        }
      }
      bool stopped = false;
#pragma unroll
      for (int u = 0; u < kU; ++u) {
        if (es[u] < 0) continue;
        if (CHECK_STOP && stop()) { stopped = true; break; }
        f(keys[u], NUM ? sh->av[es[u]] * vals[u] : VT(0));
      }
      if (CHECK_STOP && stopped) break;
    }
    __syncthreads();
  }
}

// Dispatch: flattened load-balanced loop (flat, short B rows) or the VW-lanes-per-A-entry loop.
// GMAX: the row group's lane count (TPR).  CTA-per-row groups in flat mode use
// for_each_product_block instead (see the callers).
template <bool NUM, bool CHECK_STOP, typename VT, int GMAX, typename F, typename S>
__device__ __forceinline__ void products(bool flat, const int64_t* __restrict__ a_rpt,
                                         const int32_t* __restrict__ a_col, const VT* __restrict__ a_val,
                                         const int64_t* __restrict__ b_rpt, const int32_t* __restrict__ b_col,
                                         const VT* __restrict__ b_val, int row, int t, int tpr, int vwl, F&& f,
                                         S&& stop, int long_len, int* deferred) {
  // flat only for row groups of <= 32 lanes: in CTA-per-row groups, batches of 32 consecutive A
  // non-zeros per warp leave most warps idle on rows with a few hundred non-zeros (measured)
  if (flat && GMAX <= 32)
    for_each_product_flat<NUM, CHECK_STOP, VT, (GMAX < 32 ? GMAX : 32)>(a_rpt, a_col, a_val, b_rpt, b_col, b_val, row,
                                                                       t, tpr, f, stop, long_len, deferred);
  else
    for_each_product<NUM, CHECK_STOP, VT>(a_rpt, a_col, a_val, b_rpt, b_col, b_val, row, t, tpr, vwl, f, stop,
                                          long_len, deferred);
}

// Second pass (CTA-wide, every thread of the CTA must call it): the A row is rescanned in
// chunks of kLongChunk entries; entries whose B row is longer than long_len go to a shared
// list (s_list: kLongChunk ints, s_cnt: one int; s_cnt must be 0 before pass 1 and is set by
// pass 1 when it defers a row, otherwise this pass returns at once).  The listed B rows are then
// walked flattened: their lengths are scanned into bf->incl and every thread strides the
// concatenated products, so a chunk with many long rows keeps all tpr threads' gathers in flight
// instead of walking the rows one after another (R-MAT hub rows: measured 40x on cluster rows).
// WSYNC (private-accumulator rows, where the lanes of a sub-group must hold distinct columns of
// one B row) walks the listed rows one at a time instead.  A stopped (CHECK_STOP) thread keeps
// hitting barriers.
constexpr int kLongChunk = 256;
template <bool NUM, bool CHECK_STOP, typename VT, bool WSYNC = false, typename BF, typename F, typename S>
__device__ __forceinline__ void for_long_products(const int64_t* __restrict__ a_rpt, const int32_t* __restrict__ a_col,
                                                  const VT* __restrict__ a_val, const int64_t* __restrict__ b_rpt,
                                                  const int32_t* __restrict__ b_col, const VT* __restrict__ b_val,
                                                  bool active, int row, int t, int tpr, int long_len, int* s_list,
                                                  int* s_cnt, BF* bf, F&& f, S&& stop, int part = 0,
                                                  int nparts = 1) {
  const long long a0 = active ? __ldg(a_rpt + row) : 0;
  const int32_t* __restrict__ ac = a_col + a0;
  __syncthreads();  // s_cnt doubles as the "some sub-group deferred a row" flag of pass 1
  if (*(volatile int*)s_cnt == 0) return;  // CTA-uniform
  const int na = active ? (int)(__ldg(a_rpt + row + 1) - a0) : 0;
  __syncthreads();
  if (t == 0) *s_cnt = 0;
  __syncthreads();
  for (int c = 0; c < na; c += kLongChunk) {  // na is CTA-uniform
    bool added = false;
    for (int e = t; e < kLongChunk && c + e < na; e += tpr) {
      if (nparts > 1 && (c + e) % nparts != part) continue;  // cluster: CTA `part` takes its share
      const int kk = __ldg(ac + c + e);
      if (__ldg(b_rpt + kk + 1) - __ldg(b_rpt + kk) > long_len) {
        s_list[atomicAdd(s_cnt, 1)] = c + e;
        added = true;
      }
    }
    if (__syncthreads_count(added) == 0) continue;  // no long row in this chunk: one barrier
    const int n = *s_cnt;
    if constexpr (WSYNC) {
      for (int i = 0; i < n; ++i) {
        const int j = s_list[i];
        const int kk = __ldg(ac + j);
        const VT av = NUM ? __ldg(a_val + a0 + j) : VT(0);
        const long long b0 = __ldg(b_rpt + kk);
        int len = (int)(__ldg(b_rpt + kk + 1) - b0);
        if (CHECK_STOP && stop()) len = 0;
        const int32_t* __restrict__ bc = opaque(b_col + b0);
        const VT* __restrict__ bv = NUM ? opaque(b_val + b0) : nullptr;
#pragma unroll 1
        for (int q = t; q < len; q += tpr) f(__ldg(bc + q), NUM ? av * __ldg(bv + q) : VT(0));
        __syncwarp();
      }
    } else {
      // listed rows' (start, value, length) -> shared; inclusive scan of the lengths by warps
      const int lane = t & 31, wid = t >> 5, nw = tpr >> 5;
      for (int i = t; i < n; i += tpr) {
        const int j = s_list[i];
        const int kk = __ldg(ac + j);
        const long long b0 = __ldg(b_rpt + kk);
        bf->b0[i] = b0;
        bf->incl[i] = (int)(__ldg(b_rpt + kk + 1) - b0);
        if (NUM) bf->av[i] = __ldg(a_val + a0 + j);
      }
      __syncthreads();
      for (int blk = wid; blk * 32 < n; blk += nw) {
        const int e = blk * 32 + lane;
        int v = e < n ? bf->incl[e] : 0;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
          const int y = __shfl_up_sync(0xffffffffu, v, o);
          if (lane >= o) v += y;
        }
        if (e < n) bf->incl[e] = v;
      }
      __syncthreads();
      int addv[kLongChunk / 64 + 1];  // per-thread fix-ups for its elements (n <= kLongChunk)
#pragma unroll
      for (int u = 0; u < kLongChunk / 64 + 1; ++u) {
        const int e = t + u * tpr;
        int add = 0;
        if (e < n)
          for (int b = 0; b < (e >> 5); ++b) add += bf->incl[b * 32 + 31];
        addv[u] = add;
      }
      __syncthreads();
#pragma unroll
      for (int u = 0; u < kLongChunk / 64 + 1; ++u) {
        const int e = t + u * tpr;
        if (e < n) bf->incl[e] += addv[u];
      }
      __syncthreads();
      const int P = bf->incl[n - 1];
      int e = 0;
      {  // first entry with incl > t (binary search), then advance monotonically with p
        int lo = 0, hi = n - 1;
        while (lo < hi) {
          const int mid = (lo + hi) >> 1;
          if (bf->incl[mid] <= t) lo = mid + 1; else hi = mid;
        }
        e = lo;
      }
#pragma unroll 1
      for (int p = t; p < P; p += tpr) {
        while (bf->incl[e] <= p) ++e;
        const int start = e ? bf->incl[e - 1] : 0;
        const long long q = bf->b0[e] + (p - start);
        const int key = __ldg(b_col + q);
        const VT v = NUM ? __ldg(b_val + q) : VT(0);
        if (CHECK_STOP && stop()) break;
        f(key, NUM ? bf->av[e] * v : VT(0));
      }
    }
    __syncthreads();
    if (t == 0) *s_cnt = 0;
    __syncthreads();
  }
}

// Warp-aggregated per-group accumulation into shared counters (64-bit shared atomics are
// CAS loops on sm_100a, so each distinct group of the warp issues one atomic per counter).
__device__ __forceinline__ unsigned long long warp_sum_u64(unsigned long long x) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) x += __shfl_xor_sync(0xffffffffu, x, o);
  return x;
}
__device__ __forceinline__ unsigned long long warp_max_u64(unsigned long long x) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    const unsigned long long y = __shfl_xor_sync(0xffffffffu, x, o);
    x = y > x ? y : x;
  }
  return x;
}
template <int NV>
__device__ __forceinline__ void warp_group_add(bool valid, int g, const unsigned long long (&v)[NV],
                                               unsigned long long* const (&dst)[NV]) {
  const int lane = threadIdx.x & 31;
  unsigned todo = __ballot_sync(0xffffffffu, valid);
  while (todo) {
    const int leader = __ffs(todo) - 1;
    const int gl = __shfl_sync(0xffffffffu, g, leader);
    const bool mine = valid && g == gl;
    todo &= ~__ballot_sync(0xffffffffu, mine);
#pragma unroll
    for (int i = 0; i < NV; ++i) {
      const unsigned long long x = warp_sum_u64(mine ? v[i] : 0ull);
      if (lane == leader) atomicAdd(dst[i] + gl, x);
    }
  }
}

// Row-group collectives: TPR <= 32 -> lanes of one warp (shuffles with width TPR);
// TPR > 32 -> the whole CTA (one row per CTA), ws = >= 33 ints of shared scratch.
template <int TPR>
struct Grp {
  // lanes of this row group inside its warp (TPR < 32), so rows sharing a warp may diverge
  static __device__ __forceinline__ unsigned mask() {
    if constexpr (TPR >= 32) return 0xffffffffu;
    else return ((1u << TPR) - 1u) << ((threadIdx.x & 31) & ~(TPR - 1));
  }
  static __device__ __forceinline__ void sync() {
    if constexpr (TPR <= 32) __syncwarp(mask()); else __syncthreads();
  }
  static __device__ __forceinline__ int lane() { return threadIdx.x % TPR; }

  // exclusive prefix of v over the group; *total receives the group sum.
  static __device__ __forceinline__ long long excl_scan(long long v, long long* total, long long* ws) {
    if constexpr (TPR <= 32) {
      long long x = v;
#pragma unroll
      for (int d = 1; d < TPR; d <<= 1) {
        long long y = __shfl_up_sync(mask(), x, d, TPR);
        if (lane() >= d) x += y;
      }
      *total = __shfl_sync(mask(), x, TPR - 1, TPR);
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

  // group min of mn and max of mx, written to out[0], out[1] (visible to the whole group on
  // return); out must be per-group shared memory.
  static __device__ __forceinline__ void minmax(int mn, int mx, int* out) {
    if constexpr (TPR <= 32) {
#pragma unroll
      for (int o = TPR / 2; o > 0; o >>= 1) {
        mn = min(mn, __shfl_xor_sync(mask(), mn, o, TPR));
        mx = max(mx, __shfl_xor_sync(mask(), mx, o, TPR));
      }
      if (lane() == 0) { out[0] = mn; out[1] = mx; }
      __syncwarp(mask());
    } else {
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) {
        mn = min(mn, __shfl_xor_sync(0xffffffffu, mn, o));
        mx = max(mx, __shfl_xor_sync(0xffffffffu, mx, o));
      }
      if (threadIdx.x == 0) { out[0] = INT_MAX; out[1] = -1; }
      __syncthreads();
      if ((threadIdx.x & 31) == 0) { atomicMin(out, mn); atomicMax(out + 1, mx); }
      __syncthreads();
    }
  }

  // 32-bit group sum (REDUX on full warps); the result is valid on every thread of the group.
  static __device__ __forceinline__ int sum32(int v, int* ws32) {
    if constexpr (TPR < 32) {
#pragma unroll
      for (int o = TPR / 2; o > 0; o >>= 1) v += __shfl_xor_sync(mask(), v, o, TPR);
      return v;
    } else if constexpr (TPR == 32) {
      return __reduce_add_sync(0xffffffffu, v);
    } else {
      const int w = __reduce_add_sync(0xffffffffu, v);
      if (threadIdx.x == 0) *ws32 = 0;
      __syncthreads();
      if ((threadIdx.x & 31) == 0) atomicAdd(ws32, w);
      __syncthreads();
      return *ws32;
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
  int long_len;            // CTA-per-row groups: B rows longer than this are walked by the CTA
  int flat;                // 1: load-balanced flattened product loop (short B rows)
  const int2* rlohi;       // column span [lo_i, hi_i] of each row of C, or null (paper hash only)
  // optimistic group
  int32_t* overflow_rows; int* overflow_count; int fill_limit;
  // global fallback
  int* slab; long long slab_T; const int64_t* nprod; long long n;
  const int* dev_count;    // extra rows from overflow list (device count), may be null
  const int32_t* overflow2_rows;  // global kernel: rows that overflowed the cluster table
  const int* dev_count2;
  unsigned* rbits; long long rwcap;  // range rows: pattern bitmap, rwcap words per row of the group
  int l1_words;            // rank-count kernels: level-1 words (>= n/1024 + 1)
  int* err_flags;          // rank-count kernels: inconsistent-input flag (DevAcc::err_flags)
};

struct NumArgs {
  const int64_t* a_rpt; const int32_t* a_col; const void* a_val;
  const int64_t* b_rpt; const int32_t* b_col; const void* b_val;
  const int32_t* rows; long long nrows;
  const int64_t* c_rpt; int32_t* c_col; void* c_val;
  int vw_log2;
  int long_len;
  int flat;                // 1: load-balanced flattened product loop (short B rows)
  const int2* rlohi;       // column span of each row of C, or null (paper hash only)
  int priv_ok;             // B rows strictly increasing: private per-sub-group accumulators allowed
  int* err_flags;
  // global fallback
  void* slab; long long slab_T; long long slab_stride; long long max_nnz; long long bitmap_words;
  const unsigned* rbits; long long rwcap;  // range rows: symbolic pattern bitmap (same row order)
  int l1_words;            // CTA-per-row groups: level-1 words of the two-level rank (>= n/1024 + 1)
  unsigned long long* prof;  // diagnostics (SPGEMM_PROF_GROUP): per CTA row, %globaltimer at phase ends
  const int64_t* nprod;      // batched kernels: n_prod_i of every row (step (1))
  int* row_counter;          // cluster groups: dynamic row counter (zeroed by spgemm_numeric)
};

__device__ __forceinline__ unsigned long long gtimer() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}

cudaError_t launch_nprod_group(cudaStream_t s, long long m, long long k, const int64_t* a_rpt,
                               const int32_t* a_col, const int64_t* b_rpt, const int32_t* b_col, int2* bmm, int4* binfo,
                               int64_t* nprod, int2* rlohi, uint8_t* grp, int64_t* c_rpt, DevAcc* acc, Bounds b,
                               int32_t* defer_a, int32_t* defer_b, int* nlaunch);
cudaError_t launch_group_stats(cudaStream_t s, long long m, const uint8_t* grp1, const uint8_t* grp2,
                               const int64_t* nprod, const int64_t* a_rpt, const int64_t* c_rpt, DevAcc* acc);
cudaError_t launch_group_scatter(cudaStream_t s, long long m, const uint8_t* grp, Offsets off,
                                 int* cursor, int32_t* perm);
// Step-(6) selection of the batched numeric rows (kernels_esc.cu): rows of symbolic groups
// kEscSymLo..kEscSymHi with 100 * n_prod_i <= pct * nnz_i go to group kNumEscBase + g1 - kEscSymLo.
struct EscSel {
  const int64_t* nprod;  // null: off
  int pct;
  unsigned groups;       // bit g: symbolic group g may take the ESC kernels
};
cudaError_t launch_scan_and_group(cudaStream_t s, long long m, int64_t* c_rpt, const uint8_t* grp1,
                                  uint8_t* grp2, DevAcc* acc, Bounds b, EscSel esc,
                                  long long* tile_ws, int* nlaunch);
size_t scan_workspace_bytes(long long m);
// host_acc: pinned host copy of acc written by the kernel at its end (nullptr: none)
cudaError_t launch_scan_small(cudaStream_t s, long long m, int64_t* c_rpt, DevAcc* acc, DevAcc* host_acc);
cudaError_t launch_validate(cudaStream_t s, long long m, long long k, long long n, const int64_t* a_rpt,
                            const int32_t* a_col, const int64_t* b_rpt, const int32_t* b_col, int* err);
cudaError_t launch_partition(cudaStream_t s, long long m, const int64_t* a_rpt, const int32_t* a_col,
                             const int64_t* b_rpt, int64_t* nprod_scan, long long* tile_ws,
                             int nparts, int64_t* splits_dev, int* nlaunch);

cudaError_t launch_symbolic_group(cudaStream_t s, int group, const SymArgs& a, int num_sms);
cudaError_t launch_symbolic_global(cudaStream_t s, const SymArgs& a, int grid);
cudaError_t launch_numeric_group(cudaStream_t s, int group, bool fp64, const NumArgs& a);
cudaError_t launch_numeric_global(cudaStream_t s, bool fp64, const NumArgs& a, int grid);
cudaError_t launch_numeric_rankacc(cudaStream_t s, int group, bool fp64, const NumArgs& a);
int rankacc_smem_bytes(int group, bool fp64, int l1_words);
cudaError_t launch_symbolic_rankcnt(cudaStream_t s, int group, const SymArgs& a);
int rankcnt_smem_bytes(int group, int l1_words);
// Rank-big kernel variants: 0 = level-2 bitmap and prefix in a per-CTA global slab (1024 threads);
// 1 = in shared memory, rows of <= kRankBigSharedL2 output entries (numeric group 10, 1024
// threads); 2 = in shared memory, rows of <= kRankMidSharedL2 entries (numeric group 9, 512
// threads, two CTAs per SM)
constexpr int kRankBigSharedL2 = 24576;
constexpr int kRankMidSharedL2 = 8192;
cudaError_t launch_numeric_rankbig(cudaStream_t s, bool fp64, const NumArgs& a, int grid, int variant);
// rank kernels with the output reduced straight into C (no vals / keys arrays in shared memory):
// numeric group 9 at 512 threads, two CTAs per SM; groups 3-8 at their kRankNum shapes
cudaError_t launch_numeric_rankout(cudaStream_t s, int group, bool fp64, const NumArgs& a);
int rankout_smem_bytes(int group, bool fp64, int l1_words);
cudaError_t launch_symbolic_tiny(cudaStream_t s, int group, const SymArgs& a);
cudaError_t launch_small_symbolic(cudaStream_t s, long long m, long long k, const int64_t* a_rpt, const int32_t* a_col,
                                  const int64_t* b_rpt, const int32_t* b_col, int64_t* c_cnt, int64_t* nprod,
                                  DevAcc* acc);
cudaError_t launch_small_numeric(cudaStream_t s, bool fp64, const NumArgs& a, long long m);
cudaError_t launch_numeric_tiny(cudaStream_t s, int group, bool fp64, const NumArgs& a);
int rankbig_smem_bytes(bool fp64, int l1_words, int variant = 0);
cudaError_t launch_symbolic_cluster(cudaStream_t s, const SymArgs& a, const int32_t* rows, const int* count,
                                    int32_t* overflow2, int* count2, int fill_limit, int max_rows);
cudaError_t launch_numeric_cluster(cudaStream_t s, bool fp64, int cs, const NumArgs& a, int* nclusters_out);
cudaError_t launch_symbolic_range(cudaStream_t s, const SymArgs& a, int rmax, int num_sms);
cudaError_t launch_numeric_range(cudaStream_t s, bool fp64, const NumArgs& a, int rmax, int num_sms);
cudaError_t launch_brow_bits(cudaStream_t s, long long k, const int64_t* b_rpt, const int32_t* b_col,
                             const int2* bmm, unsigned* bbits, int bw, int* wmax, int num_sms);
cudaError_t launch_symbolic_range_bits(cudaStream_t s, const SymArgs& a, const unsigned* bbits, int bw,
                                       const int2* bmm, const int* wmax, int num_sms);
int range_warps(long long per_warp, long long budget_default = kRangeSmemBudget);
int range_rcap(long long rmax);
int range_wcap(long long rmax);
int cluster_capacity_sym();
cudaError_t launch_symbolic_batch(cudaStream_t s, int group, const SymArgs& a);
cudaError_t launch_numeric_esc(cudaStream_t s, int sym_group, bool fp64, const NumArgs& a);
bool numeric_esc_supported(int sym_group, bool fp64);
int wsort_max_group();
cudaError_t launch_symbolic_wsort(cudaStream_t s, int sym_group, const SymArgs& a);
cudaError_t launch_numeric_wsort(cudaStream_t s, int sym_group, bool fp64, const NumArgs& a);
int cluster_capacity_num();

}  // namespace spg
