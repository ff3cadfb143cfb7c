// kernels_rankacc.cu — CTA-per-row kernels for wide-span (graph) rows that index the row's
// table by the RANK of the column (B200 addition): symbolic count (step 3) and
// numeric accumulate + gather + sort (step 7).
//
// The paper's numeric phase inserts every product's column into a hash table
// (Alg. 5), adds the value into a parallel value table, then gathers the occupied slots and sorts
// them by a comparison rank; the symbolic phase counts the distinct keys of the same table
// (PAPER.md:130-155).  An entry's final position is rank(key) = #distinct columns of row i below
// key.  For rows whose column span is wide and sparse (power-law graphs: R-MAT, webbase — products
// ~ output entries, so the 2x-oversized hash tables are nearly all fixed cost) these kernels build
// that rank FIRST, from a two-level bitmap of the row's columns over its exact span [lo_i, hi_i]
// (computed with n_prod in step (1)), and use it as a collision-free, order-preserving hash:
//
//   (i)   metadata: the row's A non-zeros (<= MC*TPR), MC consecutive ones per thread: col_A,
//         val_A, rpt_B pair; block scan of the B-row lengths (Alg. 3/4's product enumeration,
//         flattened) and, per 32-product block, the A entry holding its first product (a product
//         finds its entry with one lookup and a short forward walk instead of a binary search);
//   (ii)  gather: thread t takes products t, t+TPR, ... (<= KP of them, held in registers; all
//         gathers of b_col/b_val issued before use) and sets level-1 bit (key-lo)>>5 — "this
//         32-column block is non-empty" — with a shared atomicOr;
//   (iii) prefix popcount of level 1 -> compact index of every non-empty block;
//   (iv)  each product sets its bit in the level-2 word of its block;
//   symbolic: nnz_i = popcount of level 2 (the count of inserted keys).
//   numeric:
//   (v)   prefix popcount of level 2 -> rank(key) = pre2[b] + popc(fine[b] & below(key));
//   (vi)  vals[rank] += a_ik * b_kj (shared atomic add, working precision),
//         keys[rank] = key (idempotent store);
//   (vii) the row is compact and sorted: coalesced write of keys/vals to C.
//
// No probing, no -1 initialisation of a 2x-oversized table, no compaction or sort pass; O(n_prod
// + R_i/1024) work per row.  Rows with more than MC*TPR A non-zeros or more than KP*TPR products
// walk their products with the chunked block loop once per pass (re-gathering; identical result).
// The paper's hash kernels (kernels_symbolic.cu, kernels_numeric.cu) remain for rows without a
// column span (range hash disabled), for the forced-group paths and as the ablation
// (SPGEMM_OPT_RANK_ACC = 0).
#include <climits>
#include <type_traits>

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

__device__ __forceinline__ int popc4(uint4 x) { return __popc(x.x) + __popc(x.y) + __popc(x.z) + __popc(x.w); }

#ifndef SPG_L1_SWIZZLE
#define SPG_L1_SWIZZLE 1
#endif
// Level-1 word w (and its prefix) lives at l1sw(w): bits 2-4 XOR bits 5-7.  The bank of a word is
// bits 0-4 of its index, i.e. bits 10-14 of the column offset, which are biased on R-MAT (a 1 with
// p = 0.4 per bit); XOR with the next bits evens the banks out.  Groups of 4 words stay together
// (uint4 sweeps); arrays are padded to 32 words.
__device__ __forceinline__ int l1sw(int w) { return SPG_L1_SWIZZLE ? w ^ (((w >> 5) & 7) << 2) : w; }
__host__ __device__ constexpr int l1_pad(int w) { return SPG_L1_SWIZZLE ? (w + 31) & ~31 : (w + 3) & ~3; }

// Exclusive prefix popcount of words[0..W) (W rounded up to 4 words, the tail zero) into pre
// (u16, may be null); returns the total.  One contiguous run of uint4 per thread.  SW: words and
// pre are laid out by l1sw (level 1).
template <int TPR, bool SW = false>
__device__ __forceinline__ int prefix_popc(const unsigned* words, int W, uint16_t* pre, int* ws32) {
  const int W4 = (W + 3) >> 2;
  const int per = (W4 + TPR - 1) / TPR;
  const int v0 = min(W4, (int)threadIdx.x * per), v1 = min(W4, v0 + per);
  const uint4* w4 = reinterpret_cast<const uint4*>(words);
  auto ph = [](int v) { return SW ? l1sw(4 * v) >> 2 : v; };
  int loc = 0;
  for (int v = v0; v < v1; ++v) loc += popc4(w4[ph(v)]);
  int total;
  int run = cta_scan32<TPR>(loc, &total, ws32);
  if (pre) {
    for (int v = v0; v < v1; ++v) {
      const uint4 x = w4[ph(v)];
      ushort4 o;
      o.x = (unsigned short)run; run += __popc(x.x);
      o.y = (unsigned short)run; run += __popc(x.y);
      o.z = (unsigned short)run; run += __popc(x.z);
      o.w = (unsigned short)run; run += __popc(x.w);
      reinterpret_cast<ushort4*>(pre)[ph(v)] = o;
    }
  }
  return total;
}

// u32 variant (prefix values above 65535; `global`: the words live in a global slab, read via L2)
template <int TPR, bool SW = false>
__device__ __forceinline__ int prefix_popc32(const unsigned* words, int W, unsigned* pre, int* ws32, bool global) {
  const int W4 = (W + 3) >> 2;
  const int per = (W4 + TPR - 1) / TPR;
  const int v0 = min(W4, (int)threadIdx.x * per), v1 = min(W4, v0 + per);
  const uint4* w4 = reinterpret_cast<const uint4*>(words);
  auto ph = [](int v) { return SW ? l1sw(4 * v) >> 2 : v; };
  auto ld = [&](int v) { return global ? __ldcg(w4 + ph(v)) : w4[ph(v)]; };
  int loc = 0;
  for (int v = v0; v < v1; ++v) loc += popc4(ld(v));
  int total;
  int run = cta_scan32<TPR>(loc, &total, ws32);
  for (int v = v0; v < v1; ++v) {
    const uint4 x = ld(v);
    uint4 o;
    o.x = (unsigned)run; run += __popc(x.x);
    o.y = (unsigned)run; run += __popc(x.y);
    o.z = (unsigned)run; run += __popc(x.z);
    o.w = (unsigned)run; run += __popc(x.w);
    reinterpret_cast<uint4*>(pre)[ph(v)] = o;
  }
  return total;
}

template <int TPR>
__device__ __forceinline__ void clear_words(unsigned* words, int W) {
  uint4* w4 = reinterpret_cast<uint4*>(words);
  for (int v = threadIdx.x; v < (W + 3) >> 2; v += TPR) w4[v] = make_uint4(0u, 0u, 0u, 0u);
}

// Shared-memory layout of one row (16-byte aligned pieces); VT = value type (int: symbolic).
//   vals[UPPER] VT (numeric) | b0[ME] i64 | av[ME] VT (numeric) | incl[ME] i32 |
//   keys[UPPER] i32 (numeric) | fine[UPPER] u32 | bstart[KP*TPR/32+1] i32 | l1[L1W] u32 |
//   pre2[UPPER] u16 (numeric) | p1[L1W] u16 (u32 for the chunked big-row count: more than
//   65535 non-empty blocks)
// GOUT (numeric): no vals / keys arrays — values are reduced straight into the zeroed row of C
// at their rank and keys stored there (two CTAs per SM fit; numeric group 9).
template <typename VT, bool NUM, int TPR, long long UPPER, int MC, int KP, bool GOUT = false>
struct RankLayout {
  static constexpr int ME = MC * TPR;  // metadata entries
  static constexpr bool kOwnOut = NUM && !GOUT;
  static constexpr int kVals = 0;
  static constexpr int kB0 = kOwnOut ? align16((int)(UPPER * sizeof(VT))) : 0;
  static constexpr int kAv = kB0 + align16(ME * 8);
  static constexpr int kIncl = kAv + (NUM ? align16(ME * (int)sizeof(VT)) : 0);
  static constexpr int kKeys = kIncl + align16(ME * 4);
  static constexpr int kFine = kKeys + (kOwnOut ? align16((int)UPPER * 4) : 0);
  static constexpr int kBstart = kFine + align16((int)UPPER * 4);
  static constexpr int kL1 = kBstart + align16((KP * TPR / 32 + 1) * 4);
  static __host__ __device__ constexpr int pre2(int l1w) { return kL1 + align16(l1_pad(l1w) * 4); }
  static __host__ __device__ constexpr int p1(int l1w) { return pre2(l1w) + (NUM ? align16((int)UPPER * 2) : 0); }
  using P1T = std::conditional_t<(!NUM && UPPER > 16384), unsigned, uint16_t>;
  static __host__ __device__ constexpr int bytes(int l1w) { return p1(l1w) + align16(l1_pad(l1w) * (int)sizeof(P1T)); }
};

// Per-group launch shape of the rank kernels (independent of the hash groups' Table-I shapes):
// TPR threads (one row per CTA), KP products per thread held in registers (fast path: n_prod_i <=
// KP*TPR), MC A non-zeros of metadata per thread (fast path: nnz(A_i) <= MC*TPR).  Numeric groups
// are keyed by nnz_i (graph rows: n_prod_i ~ nnz_i, so KP*TPR >= the bound), symbolic groups by
// n_prod_i (KP*TPR = the bound).
struct RankCfg {
  int TPR, KP, MC;
};
// numeric: KP*TPR = the nnz bound for groups 6-8 (graph rows' n_prod_i is within ~1 % of nnz_i;
// the few rows above it take the re-walk path) — half the warps per row of KP*TPR = 2x the bound
// (R-MAT s20: groups 6-8 1.86/2.21/1.90 -> 1.73/1.69/1.82 ms); group 5 keeps 128 threads (64:
// the span-sized level-1 bitmap per CTA limits residency, 1.21 -> 1.38 ms)
constexpr RankCfg kRankNum[] = {{0, 0, 0},   {0, 0, 0},    {0, 0, 0},    {64, 4, 2},   {64, 8, 2},
                                {128, 8, 2}, {128, 12, 2}, {256, 12, 2}, {512, 12, 2}, {1024, 9, 2}};
// symbolic groups 3-4 stay on the paper hash (faster there: measured R-MAT s20 0.28/0.66 ms vs
// 0.53/0.69 ms); MC 4 measured slower than 2 for groups 5-8
constexpr RankCfg kRankSym[] = {{0, 0, 0},    {0, 0, 0},    {0, 0, 0},    {64, 4, 2},   {64, 8, 2},
                                {64, 16, 2},  {128, 16, 2}, {256, 16, 2}, {512, 16, 2}, {1024, 16, 2}};
__host__ __device__ constexpr int rankbig_l1pad_h(int l1w) { return ((l1w + 31) & ~31); }

// Adapters so rank_row reads both argument structs the same way.
struct NumView : NumArgs {
  __device__ __forceinline__ const void* a_val_ptr() const { return a_val; }
  __device__ __forceinline__ const void* b_val_ptr() const { return b_val; }
};
struct SymView : SymArgs {
  __device__ __forceinline__ const void* a_val_ptr() const { return nullptr; }
  __device__ __forceinline__ const void* b_val_ptr() const { return nullptr; }
};

#ifndef SPG_RANK_SETCHECK
#define SPG_RANK_SETCHECK 2  // read a bitmap bit before setting it: 1 always, 0 never, 2 numeric by compression
#endif
// One row, symbolic (NUM = false: writes nnz_i to c_cnt[row]) or numeric (writes the row of C).
template <typename VT, bool NUM, int TPR, long long UPPER, int KP, int MC, bool GOUT = false, typename Args>
__device__ __forceinline__ void rank_row(const Args& a, int row, unsigned char* smem_raw, int (*ws32)[32],
                                         long long* ws64) {
  using L = RankLayout<VT, NUM, TPR, UPPER, MC, KP, GOUT>;
  constexpr int ME = L::ME;
  VT* vals = reinterpret_cast<VT*>(smem_raw + L::kVals);
  long long* sb0 = reinterpret_cast<long long*>(smem_raw + L::kB0);
  VT* sav = reinterpret_cast<VT*>(smem_raw + L::kAv);
  int* sincl = reinterpret_cast<int*>(smem_raw + L::kIncl);
  int* keys = reinterpret_cast<int*>(smem_raw + L::kKeys);
  unsigned* fine = reinterpret_cast<unsigned*>(smem_raw + L::kFine);
  int* bstart = reinterpret_cast<int*>(smem_raw + L::kBstart);
  unsigned* l1 = reinterpret_cast<unsigned*>(smem_raw + L::kL1);
  uint16_t* pre2 = reinterpret_cast<uint16_t*>(smem_raw + L::pre2(a.l1_words));
  using P1T = typename L::P1T;
  P1T* p1 = reinterpret_cast<P1T*>(smem_raw + L::p1(a.l1_words));

  const VT* __restrict__ av_g = static_cast<const VT*>(a.a_val_ptr());
  const VT* __restrict__ bv_g = static_cast<const VT*>(a.b_val_ptr());
  const int32_t* __restrict__ bc_g = a.b_col;
  const int t = threadIdx.x;
  const long long a0 = __ldg(a.a_rpt + row);
  const int na = (int)(__ldg(a.a_rpt + row + 1) - a0);
  const int2 rr = __ldg(a.rlohi + row);
  const int lo = rr.x;
  const int W1 = rr.y >= rr.x ? (int)(((unsigned)(rr.y - rr.x)) >> 10) + 1 : 0;  // CTA-uniform
  clear_words<TPR>(l1, l1_pad(W1));

  // (i) metadata: thread t owns A non-zeros t*MC .. t*MC+MC-1
  int lens[MC];
  int mysum = 0;
#pragma unroll
  for (int j = 0; j < MC; ++j) {
    const int e = t * MC + j;
    lens[j] = 0;
    if (e < na) {
      const int kk = __ldg(a.a_col + a0 + e);
      const long long b0 = __ldg(a.b_rpt + kk);
      lens[j] = (int)(__ldg(a.b_rpt + kk + 1) - b0);
      sb0[e] = b0;
      if constexpr (NUM) sav[e] = __ldg(av_g + a0 + e);
    }
    mysum += lens[j];
  }
  int P;
  int run = cta_scan32<TPR>(mysum, &P, ws32[0]);
  const bool fast = na <= ME && P <= KP * TPR;  // CTA-uniform
#pragma unroll
  for (int j = 0; j < MC; ++j) {
    const int e = t * MC + j;
    if (e < na) {
      const int s = run, en = run + lens[j];
      sincl[e] = en;
      if (fast)  // 32-product blocks whose first product lies in this entry
        for (int k = (s + 31) >> 5; k < ((en + 31) >> 5); ++k) bstart[k] = e;
      run = en;
    }
  }
  __syncthreads();

  int key[KP];
  VT val[KP];
  // set-if-clear: rows that compress (duplicate columns) would otherwise serialise on the same
  // words; a stale read only costs a redundant atomic.  The numeric phase knows nnz_i: rows whose
  // products are (almost) all distinct (n_prod_i <= 17/16 nnz_i: graph rows) skip the read, since
  // nearly every bit is new (CTA-uniform; R-MAT s22 numeric group 9 5.57 -> 5.39 ms).  Symbolic
  // rows always read (webbase-like rows repeat columns; their span does not tell them apart)
  bool chk = SPG_RANK_SETCHECK != 0;
  if constexpr (NUM) {
    if (SPG_RANK_SETCHECK == 2) {
      const long long nz = a.c_rpt[row + 1] - a.c_rpt[row];
      chk = (long long)P > nz + (nz >> 4);
    }
  }
  auto set_l1 = [&](int k) {
    const unsigned d = (unsigned)(k - lo);
    const unsigned bit = 1u << ((d >> 5) & 31);
    const int w = l1sw((int)(d >> 10));
    if (!chk || !(l1[w] & bit)) atomicOr(l1 + w, bit);
  };
  auto blk_of = [&](unsigned d) {
    const int w = l1sw((int)(d >> 10));
    const unsigned bit = (d >> 5) & 31;
    return (int)p1[w] + __popc(l1[w] & ((1u << bit) - 1u));
  };
  // level 2 of the blocks with compact index in [c0, c0 + UPPER) (symbolic rows with more
  // non-empty blocks than UPPER take them in chunks; numeric: c0 = 0 and nb <= UPPER)
  bool chk2 = chk;  // level 2: symbolic rows decide from level 1 (below)
  auto set_fine = [&](int k, int c0) {
    const unsigned d = (unsigned)(k - lo);
    const int b = blk_of(d) - c0;
    const unsigned bit = 1u << (d & 31);
    if ((NUM || (unsigned)b < (unsigned)UPPER) && (!chk2 || !(fine[b] & bit))) atomicOr(fine + b, bit);
  };
  int32_t* cc_row = nullptr;
  VT* cv_row = nullptr;
  if constexpr (NUM && GOUT) {
    cc_row = a.c_col + a.c_rpt[row];
    cv_row = static_cast<VT*>(a.c_val) + a.c_rpt[row];
  }
  auto accumulate = [&](int k, VT v) {
    const unsigned d = (unsigned)(k - lo);
    const int b = blk_of(d);
    const int r = (int)pre2[b] + __popc(fine[b] & ((1u << (d & 31)) - 1u));
    if constexpr (GOUT) {
      atomicAdd(cv_row + r, v);  // red.global.add into the zeroed row (working precision)
      cc_row[r] = k;
    } else {
      atomicAdd(vals + r, v);
      keys[r] = k;
    }
  };
  BlockFlat<VT, TPR>* bf = reinterpret_cast<BlockFlat<VT, TPR>*>(sb0);
  static_assert(sizeof(BlockFlat<VT, TPR>) <= (size_t)(L::kKeys - L::kB0) + 16, "block-flat view");
  auto walk = [&](auto&& f) {  // slow path: chunked block loop over all products (re-gathers)
    for_each_product_block<NUM, false, VT, TPR>(a.a_rpt, a.a_col, av_g, a.b_rpt, bc_g, bv_g, true, row, t, bf, ws64,
                                                f, NoStopR{});
  };

  // (ii) gather + level 1
  if (fast) {
#pragma unroll
    for (int u = 0; u < KP; ++u) {
      const int p = t + u * TPR;
      key[u] = -1;
      if (p < P) {
        int e = bstart[p >> 5];
        while (sincl[e] <= p) ++e;
        const long long q = sb0[e] + (p - (e ? sincl[e - 1] : 0));
        key[u] = __ldg(bc_g + q);
        if constexpr (NUM) val[u] = sav[e] * __ldg(bv_g + q);
      }
    }
    int u0 = 0;
    if constexpr (!NUM) {
      if (SPG_RANK_SETCHECK == 2) {
        // symbolic: the first product of every thread sets its level-1 bit after reading it; if
        // more than 1 in 32 of these found the bit already set the row repeats blocks and keeps
        // reading, else (a graph row) the rest set their bits unread
        bool hit = false;
        if (key[0] >= 0) {
          const unsigned d = (unsigned)(key[0] - lo);
          const unsigned bit = 1u << ((d >> 5) & 31);
          const int w = l1sw((int)(d >> 10));
          hit = (l1[w] & bit) != 0;
          if (!hit) atomicOr(l1 + w, bit);
        }
        chk = 32 * __syncthreads_count(hit) > TPR;
        u0 = 1;
      }
    }
#pragma unroll
    for (int u = 0; u < KP; ++u)
      if (u >= u0 && key[u] >= 0) set_l1(key[u]);
  } else {
    walk([&](int k, VT) { set_l1(k); });
  }
  __syncthreads();
  // (iii) compact index of the non-empty 32-column blocks
  int nb;
  if constexpr (sizeof(P1T) == 4) nb = prefix_popc32<TPR, true>(l1, W1, p1, ws32[1], false);
  else nb = prefix_popc<TPR, true>(l1, W1, p1, ws32[1]);
  // symbolic: nearly one non-empty 32-column block per product (nb >= 7/8 n_prod_i: a graph row)
  // means level-2 bits are almost all new, so they are set without reading them first
  if constexpr (!NUM) {
    if (SPG_RANK_SETCHECK == 2) chk2 = 8LL * nb < 7LL * P;
  }
  // CTA-uniform; numeric: false only for inconsistent input (the symbolic count bounds nb)
  const bool ok = !NUM || nb <= (int)UPPER;
  auto level2 = [&](int c0) {
    if (fast) {
#pragma unroll
      for (int u = 0; u < KP; ++u)
        if (key[u] >= 0) set_fine(key[u], c0);
    } else {
      walk([&](int k, VT) { set_fine(k, c0); });
    }
  };
  if (ok) clear_words<TPR>(fine, min(nb, (int)UPPER));
  __syncthreads();
  // (iv) level 2
  if (ok) level2(0);
  __syncthreads();
  if constexpr (!NUM) {
    // symbolic: nnz_i = number of distinct columns = popcount of level 2, chunk by chunk
    int n = prefix_popc<TPR>(fine, min(nb, (int)UPPER), nullptr, ws32[0]);
    for (int c0 = (int)UPPER; c0 < nb; c0 += (int)UPPER) {  // CTA-uniform
      __syncthreads();
      clear_words<TPR>(fine, min(nb - c0, (int)UPPER));
      __syncthreads();
      level2(c0);
      __syncthreads();
      n += prefix_popc<TPR>(fine, min(nb - c0, (int)UPPER), nullptr, ws32[(c0 / (int)UPPER) & 1]);
    }
    if (t == 0) a.c_cnt[row] = n;
  } else {
    const long long c0 = a.c_rpt[row];
    const int cn = (int)(a.c_rpt[row + 1] - c0);
    // (v) rank of every block's first key
    const int n_total = ok ? prefix_popc<TPR>(fine, nb, pre2, ws32[0]) : 0;
    if (t == 0 && n_total != cn) atomicOr(a.err_flags, 2);
    const int nw = ok ? min(n_total, cn) : 0;
    if constexpr (GOUT) {
      for (int r = t; r < nw; r += TPR) cv_row[r] = VT(0);
    } else {
      for (int r = t; r < nw; r += TPR) vals[r] = VT(0);
    }
    __syncthreads();
    // (vi) accumulate at the rank (GOUT writes C directly: only when the counts agree, so an
    // inconsistent input cannot write past the row; err_flags bit 1 is raised above)
    if (ok && (!GOUT || n_total == cn)) {
      if (fast) {
#pragma unroll
        for (int u = 0; u < KP; ++u)
          if (key[u] >= 0) accumulate(key[u], val[u]);
      } else {
        walk([&](int k, VT v) { accumulate(k, v); });
      }
    }
    __syncthreads();
    // (vii) sorted, compact row -> C (coalesced)
    if constexpr (!GOUT) {
      int32_t* __restrict__ cc = a.c_col + c0;
      VT* __restrict__ cv = static_cast<VT*>(a.c_val) + c0;
      for (int r = t; r < nw; r += TPR) {
        cc[r] = keys[r];
        cv[r] = vals[r];
      }
    }
  }
}

template <typename VT>
constexpr int rankbig_smem_bytes_v(int l1w) { return 2 * rankbig_l1pad_h(l1w) * 4 + (int)sizeof(BlockFlat<VT, 1024, 2048>); }
// dynamic shared memory of k_num_rankbig<VT, SL2, TPR>
template <typename VT, int SL2, int TPR>
constexpr int rankbig_smem_bytes_t(int l1w) {
  return 2 * rankbig_l1pad_h(l1w) * 4 + (SL2 > 0 ? align16((int)sizeof(BlockFlat<VT, TPR, 2048>)) + 6 * SL2
                                                : (int)sizeof(BlockFlat<VT, TPR, 2048>));
}

// 40 registers (1536 threads per SM) for fp32 / symbolic; fp64 values need 64 (no spills)
// (KP > 8 products per thread: 1280 threads, ~48 registers)
template <int TPR, int VB, int KP = 8>
constexpr int rank_min_blocks() { return TPR >= 1024 ? 1 : (VB > 4 ? 1024 : KP > 8 ? 1280 : 1536) / TPR; }

template <typename VT, int TPR, long long UPPER, int KP, int MC>
__global__ __launch_bounds__(TPR, rank_min_blocks<TPR, sizeof(VT), KP>()) void k_num_rankacc(NumArgs a) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  __shared__ int ws32[2][32];
  __shared__ long long ws64[33];
  rank_row<VT, true, TPR, UPPER, KP, MC>(static_cast<const NumView&>(a), a.rows[blockIdx.x], smem_raw, ws32, ws64);
}

// Numeric group 9 with the products in registers and the output reduced into C: TPR 512, two
// CTAs per SM (the one-CTA-per-SM kernel idles the SM at every per-row barrier)
template <typename VT, int TPR, long long UPPER, int KP, int MC>
__global__ __launch_bounds__(TPR, rank_min_blocks<TPR, sizeof(VT), KP>()) void k_num_rankout(NumArgs a) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  __shared__ int ws32[2][32];
  __shared__ long long ws64[33];
  rank_row<VT, true, TPR, UPPER, KP, MC, true>(static_cast<const NumView&>(a), a.rows[blockIdx.x], smem_raw, ws32,
                                               ws64);
}

template <int TPR, long long UPPER, int KP, int MC>
__global__ __launch_bounds__(TPR, rank_min_blocks<TPR, 4>()) void k_sym_rankcnt(SymArgs a) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  __shared__ int ws32[2][32];
  __shared__ long long ws64[33];
  rank_row<int, false, TPR, UPPER, KP, MC>(static_cast<const SymView&>(a), a.rows[blockIdx.x], smem_raw, ws32, ws64);
}

template <typename K>
cudaError_t prepare(K kernel, int smem, PerDevice& cache) {
  auto& configured = cache.here();
  if (smem > configured.load()) {
    cudaError_t e = cudaFuncSetAttribute(kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    if (e != cudaSuccess) return e;
    // the rows' B gathers are scattered (L1 hit rates ~30%): give the SM's memory to the tables
    e = cudaFuncSetAttribute(kernel, cudaFuncAttributePreferredSharedMemoryCarveout, 100);
    if (e != cudaSuccess) return e;
    configured.store(smem);
  }
  return cudaSuccess;
}

template <typename VT, int G>
cudaError_t launch_rankacc_k(cudaStream_t s, const NumArgs& a) {
  constexpr RankCfg c = kRankNum[G];
  constexpr long long UPPER = kNumGroups[G].upper;
  using L = RankLayout<VT, true, c.TPR, UPPER, c.MC, c.KP>;
  const int smem = L::bytes(a.l1_words);
  static PerDevice configured;
  cudaError_t e = prepare(k_num_rankacc<VT, c.TPR, UPPER, c.KP, c.MC>, smem, configured);
  if (e != cudaSuccess) return e;
  k_num_rankacc<VT, c.TPR, UPPER, c.KP, c.MC><<<(unsigned)a.nrows, c.TPR, smem, s>>>(a);
  return cudaGetLastError();
}

template <int G>
cudaError_t launch_rankcnt_k(cudaStream_t s, const SymArgs& a) {
  constexpr RankCfg c = kRankSym[G];
  constexpr long long UPPER = kSymGroups[G].upper;
  using L = RankLayout<int, false, c.TPR, UPPER, c.MC, c.KP>;
  const int smem = L::bytes(a.l1_words);
  static PerDevice configured;
  cudaError_t e = prepare(k_sym_rankcnt<c.TPR, UPPER, c.KP, c.MC>, smem, configured);
  if (e != cudaSuccess) return e;
  k_sym_rankcnt<c.TPR, UPPER, c.KP, c.MC><<<(unsigned)a.nrows, c.TPR, smem, s>>>(a);
  return cudaGetLastError();
}

// Rows above the last symbolic bound (n_prod_i > 16384, the optimistic group): exact count in one
// CTA of 1024 threads whatever the row — level 2 in chunks of kRankBigSymUpper blocks, products
// re-walked per pass — instead of the optimistic table and its cluster / global retries.
constexpr long long kRankBigSymUpper = 32768;
using RankBigSymL = RankLayout<int, false, 1024, kRankBigSymUpper, 2, 16>;
cudaError_t launch_rankcnt_big(cudaStream_t s, const SymArgs& a) {
  const int smem = RankBigSymL::bytes(a.l1_words);
  static PerDevice configured;
  cudaError_t e = prepare(k_sym_rankcnt<1024, kRankBigSymUpper, 16, 2>, smem, configured);
  if (e != cudaSuccess) return e;
  k_sym_rankcnt<1024, kRankBigSymUpper, 16, 2><<<(unsigned)a.nrows, 1024, smem, s>>>(a);
  return cudaGetLastError();
}

// output-in-C rank kernels: group 9 at 512 threads (two CTAs per SM), groups 3-8 at kRankNum
constexpr RankCfg rank_out_cfg(int g) {
  return g == 10 ? RankCfg{1024, 16, 2} : g == 9 ? RankCfg{512, 16, 2} : kRankNum[g];
}
template <typename VT, int G>
using RankOutL = RankLayout<VT, true, rank_out_cfg(G).TPR, kNumGroups[G].upper, rank_out_cfg(G).MC, rank_out_cfg(G).KP, true>;
template <typename VT, int G>
cudaError_t launch_rankout_k(cudaStream_t s, const NumArgs& a) {
  constexpr RankCfg c = rank_out_cfg(G);
  constexpr long long UPPER = kNumGroups[G].upper;
  const int smem = RankOutL<VT, G>::bytes(a.l1_words);
  static PerDevice configured;
  cudaError_t e = prepare(k_num_rankout<VT, c.TPR, UPPER, c.KP, c.MC>, smem, configured);
  if (e != cudaSuccess) return e;
  k_num_rankout<VT, c.TPR, UPPER, c.KP, c.MC><<<(unsigned)a.nrows, c.TPR, smem, s>>>(a);
  return cudaGetLastError();
}

template <typename VT>
cudaError_t launch_rankacc_v(cudaStream_t s, int group, const NumArgs& a) {
  switch (group) {
#define SPG_G(I) \
  case I: return launch_rankacc_k<VT, I>(s, a);
    SPG_G(3) SPG_G(4) SPG_G(5) SPG_G(6) SPG_G(7) SPG_G(8) SPG_G(9)
#undef SPG_G
    default: return cudaErrorInvalidValue;
  }
}

// ---------------------------------------------------------------------------------------------
// Rows above the largest CTA group (nnz_i > 8192; numeric groups 10-12): one 1024-thread CTA per
// row, persistent, rows handed out through a global counter.  Level 1 (and its u32 prefix) stays
// in shared memory; level 2 and its prefix live in a per-CTA global slab (L2-resident; up to
// 8 B per output entry); values are accumulated directly into the row of C at their rank
// (red.global.add, working precision) after the row is zeroed, keys stored there too.  Products
// are walked three times (level 1, level 2, accumulate) with the chunked block loop; the second
// and third walks re-gather B rows that the first one brought into L2.


// SL2 > 0: level 2 (u32) and its prefix (u16) in shared memory, SL2 entries each (rows of at most
// SL2 output entries: numeric groups 9-10), else both in the per-CTA global slab (L2-resident).
// TPR 512: two CTAs per SM (numeric group 9: one row's barriers no longer idle the SM).
template <typename VT, int SL2, int TPR>
__global__ __launch_bounds__(TPR, 1024 / TPR) void k_num_rankbig(NumArgs a) {
  constexpr bool SH = SL2 > 0;
  extern __shared__ __align__(16) unsigned char smem_raw[];
  __shared__ int ws32[2][32];
  __shared__ long long ws64[33];
  __shared__ int s_i;
  const int l1p = rankbig_l1pad_h(a.l1_words);
  unsigned* l1 = reinterpret_cast<unsigned*>(smem_raw);
  unsigned* p1 = l1 + l1p;
  BlockFlat<VT, TPR, 2048>* bf = reinterpret_cast<BlockFlat<VT, TPR, 2048>*>(p1 + l1p);
  unsigned* fine = SH ? reinterpret_cast<unsigned*>(reinterpret_cast<unsigned char*>(bf) + align16((int)sizeof(*bf)))
                      : reinterpret_cast<unsigned*>(static_cast<unsigned char*>(a.slab) + (long long)blockIdx.x * a.slab_stride);
  unsigned* pre2 = fine + (SH ? 0LL : a.slab_T);             // global: u32 prefix after level 2
  uint16_t* pre2s = reinterpret_cast<uint16_t*>(fine + SL2);  // shared: u16 prefix (<= SL2 entries)
  const VT* __restrict__ av_g = static_cast<const VT*>(a.a_val);
  const VT* __restrict__ bv_g = static_cast<const VT*>(a.b_val);
  const int t = threadIdx.x;
  while (true) {
    if (t == 0) s_i = atomicAdd(a.row_counter, 1);
    __syncthreads();
    const int i = s_i;
    if (i >= a.nrows) break;  // CTA-uniform
    const int row = a.rows[i];
    const int2 rr = __ldg(a.rlohi + row);
    const int lo = rr.x;
    const int W1 = rr.y >= rr.x ? (int)(((unsigned)(rr.y - rr.x)) >> 10) + 1 : 0;
    const long long c0 = a.c_rpt[row];
    const int cn = (int)(a.c_rpt[row + 1] - c0);
    int32_t* __restrict__ cc = a.c_col + c0;
    VT* __restrict__ cv = static_cast<VT*>(a.c_val) + c0;
    clear_words<TPR>(l1, l1_pad(W1));
    for (int r = t; r < cn; r += TPR) cv[r] = VT(0);
    auto walk = [&](auto&& f) {
      for_each_product_block<true, false, VT, TPR>(a.a_rpt, a.a_col, av_g, a.b_rpt, a.b_col, bv_g, true, row, t, bf,
                                                   ws64, f, NoStopR{});
    };
    auto blk_of = [&](unsigned d) {
      const int w = l1sw((int)(d >> 10));
      const unsigned bit = (d >> 5) & 31;
      return (int)p1[w] + __popc(l1[w] & ((1u << bit) - 1u));
    };
    // set-if-clear only on rows whose columns repeat (n_prod_i > 17/16 nnz_i), as in rank_row
    const bool chk = SPG_RANK_SETCHECK == 1 ||
                     (SPG_RANK_SETCHECK == 2 && (a.nprod == nullptr || a.nprod[row] > (long long)cn + (cn >> 4)));
    __syncthreads();
    walk([&](int k, VT) {
      const unsigned d = (unsigned)(k - lo);
      const unsigned bit = 1u << ((d >> 5) & 31);
      const int w = l1sw((int)(d >> 10));
      if (!chk || !(l1[w] & bit)) atomicOr(l1 + w, bit);
    });
    __syncthreads();
    const int nb = prefix_popc32<TPR, true>(l1, W1, p1, ws32[1], false);
    const bool ok = nb <= (SH ? SL2 : (int)a.slab_T);  // CTA-uniform; false only for inconsistent input
    if (ok) {
      uint4* f4 = reinterpret_cast<uint4*>(fine);
      for (int v = t; v < (nb + 3) >> 2; v += TPR) f4[v] = make_uint4(0u, 0u, 0u, 0u);
    }
    __syncthreads();
    if (ok)
      walk([&](int k, VT) {
        const unsigned d = (unsigned)(k - lo);
        atomicOr(fine + blk_of(d), 1u << (d & 31));
      });
    __syncthreads();
    int n_total = 0;
    if (ok) {
      if constexpr (SH) n_total = prefix_popc<TPR>(fine, nb, pre2s, ws32[0]);
      else n_total = prefix_popc32<TPR>(fine, nb, pre2, ws32[0], true);
    }
    if (t == 0 && n_total != cn) atomicOr(a.err_flags, 2);
    __syncthreads();
    if (ok && n_total == cn)
      walk([&](int k, VT v) {
        const unsigned d = (unsigned)(k - lo);
        const int b = blk_of(d);
        int r;
        if constexpr (SH) r = (int)pre2s[b] + __popc(fine[b] & ((1u << (d & 31)) - 1u));
        else r = (int)__ldcg(pre2 + b) + __popc(__ldcg(fine + b) & ((1u << (d & 31)) - 1u));
        atomicAdd(cv + r, v);
        cc[r] = k;
      });
    __syncthreads();
  }
}

template <typename VT, int SL2, int TPR>
cudaError_t launch_rankbig_v(cudaStream_t s, const NumArgs& a, int grid) {
  const int smem = rankbig_smem_bytes_t<VT, SL2, TPR>(a.l1_words);
  static PerDevice configured;
  cudaError_t e = prepare(k_num_rankbig<VT, SL2, TPR>, smem, configured);
  if (e != cudaSuccess) return e;
  k_num_rankbig<VT, SL2, TPR><<<grid, TPR, smem, s>>>(a);
  return cudaGetLastError();
}

constexpr int kStaticRankBytes = 2 * 32 * 4 + 33 * 8 + 1024;  // static shared + driver reserve

}  // namespace

int rankacc_smem_bytes(int group, bool fp64, int l1_words) {
  switch (group) {
#define SPG_G(I)                                                                                     \
  case I:                                                                                            \
    return kStaticRankBytes +                                                                        \
           (fp64 ? RankLayout<double, true, kRankNum[I].TPR, kNumGroups[I].upper, kRankNum[I].MC,    \
                              kRankNum[I].KP>::bytes(l1_words)                                       \
                 : RankLayout<float, true, kRankNum[I].TPR, kNumGroups[I].upper, kRankNum[I].MC,     \
                              kRankNum[I].KP>::bytes(l1_words));
    SPG_G(3) SPG_G(4) SPG_G(5) SPG_G(6) SPG_G(7) SPG_G(8) SPG_G(9)
#undef SPG_G
    default: return INT_MAX;
  }
}

int rankcnt_smem_bytes(int group, int l1_words) {
  switch (group) {
    case kSymOptimistic: return kStaticRankBytes + RankBigSymL::bytes(l1_words);
#define SPG_G(I)                                                                                  \
  case I:                                                                                         \
    return kStaticRankBytes + RankLayout<int, false, kRankSym[I].TPR, kSymGroups[I].upper,        \
                                         kRankSym[I].MC, kRankSym[I].KP>::bytes(l1_words);
    SPG_G(3) SPG_G(4) SPG_G(5) SPG_G(6) SPG_G(7) SPG_G(8) SPG_G(9)
#undef SPG_G
    default: return INT_MAX;
  }
}

int rankout_smem_bytes(int group, bool fp64, int l1_words) {
  switch (group) {
#define SPG_G(I) \
  case I: return kStaticRankBytes + (fp64 ? RankOutL<double, I>::bytes(l1_words) : RankOutL<float, I>::bytes(l1_words));
    SPG_G(3) SPG_G(4) SPG_G(5) SPG_G(6) SPG_G(7) SPG_G(8) SPG_G(9) SPG_G(10)
#undef SPG_G
    default: return INT_MAX;
  }
}

cudaError_t launch_numeric_rankout(cudaStream_t s, int group, bool fp64, const NumArgs& a) {
  if (a.nrows <= 0) return cudaSuccess;
  switch (group) {
#define SPG_G(I) \
  case I: return fp64 ? launch_rankout_k<double, I>(s, a) : launch_rankout_k<float, I>(s, a);
    SPG_G(3) SPG_G(4) SPG_G(5) SPG_G(6) SPG_G(7) SPG_G(8) SPG_G(9) SPG_G(10)
#undef SPG_G
    default: return cudaErrorInvalidValue;
  }
}

cudaError_t launch_numeric_rankacc(cudaStream_t s, int group, bool fp64, const NumArgs& a) {
  if (a.nrows <= 0) return cudaSuccess;
  return fp64 ? launch_rankacc_v<double>(s, group, a) : launch_rankacc_v<float>(s, group, a);
}

int rankbig_smem_bytes(bool fp64, int l1_words, int variant) {
  switch (variant) {
    case 1: return kStaticRankBytes + (fp64 ? rankbig_smem_bytes_t<double, kRankBigSharedL2, 1024>(l1_words)
                                            : rankbig_smem_bytes_t<float, kRankBigSharedL2, 1024>(l1_words));
    case 2: return kStaticRankBytes + (fp64 ? rankbig_smem_bytes_t<double, kRankMidSharedL2, 512>(l1_words)
                                            : rankbig_smem_bytes_t<float, kRankMidSharedL2, 512>(l1_words));
    default: return kStaticRankBytes + (fp64 ? rankbig_smem_bytes_t<double, 0, 1024>(l1_words)
                                             : rankbig_smem_bytes_t<float, 0, 1024>(l1_words));
  }
}

cudaError_t launch_numeric_rankbig(cudaStream_t s, bool fp64, const NumArgs& a, int grid, int variant) {
  if (a.nrows <= 0 || grid <= 0) return cudaSuccess;
  switch (variant) {
    case 1: return fp64 ? launch_rankbig_v<double, kRankBigSharedL2, 1024>(s, a, grid)
                        : launch_rankbig_v<float, kRankBigSharedL2, 1024>(s, a, grid);
    case 2: return fp64 ? launch_rankbig_v<double, kRankMidSharedL2, 512>(s, a, grid)
                        : launch_rankbig_v<float, kRankMidSharedL2, 512>(s, a, grid);
    default: return fp64 ? launch_rankbig_v<double, 0, 1024>(s, a, grid) : launch_rankbig_v<float, 0, 1024>(s, a, grid);
  }
}

cudaError_t launch_symbolic_rankcnt(cudaStream_t s, int group, const SymArgs& a) {
  if (a.nrows <= 0) return cudaSuccess;
  switch (group) {
    case kSymOptimistic: return launch_rankcnt_big(s, a);
#define SPG_G(I) \
  case I: return launch_rankcnt_k<I>(s, a);
    SPG_G(3) SPG_G(4) SPG_G(5) SPG_G(6) SPG_G(7) SPG_G(8) SPG_G(9)
#undef SPG_G
    default: return cudaErrorInvalidValue;
  }
}

}  // namespace spg
