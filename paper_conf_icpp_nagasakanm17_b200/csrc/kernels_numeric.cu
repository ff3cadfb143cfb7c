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
// every other (O(nnz_i^2) per row).  Here, with [lo, hi] the row's column range (a group
// min/max over the table after accumulation):
//   (c1) entries are scattered into NB buckets of width 2^shift over [lo, hi] and a thread
//        per key ranks it as bucket start + #smaller keys in the bucket (the paper's
//        comparison rank restricted to a bucket) — every bucket when range/NB <= 4
//        (banded/FEM rows), buckets of <= 8 keys in CTA-per-row groups;
//   (c4) crowded buckets of CTA-per-row groups (> 8 keys): one warp per bucket, round-robin
//        over the warps, ranks its keys by shuffle comparisons (<= 32 keys) or a per-warp
//        bitmap + popcount prefix;
//   (c2) wider ranges, sub-warp row groups (<= 128 keys): bitonic sort of the slot indices;
//   (c3) global-memory rows: bitmap over [lo, hi] + prefix popcounts.
// Keys are distinct, so every path writes the identical, sorted row.
#include <climits>

#include "spgemm_internal.cuh"

namespace spg {

namespace {

// bitmap words per warp for the (c4) rank: 4096 columns for small CTAs, 1024 for 512/1024
// threads (shared memory of the largest tables).
template <int TPR>
constexpr int kWarpBitmapWords = TPR <= 256 ? 128 : 32;

struct NoStop {
  __device__ __forceinline__ bool operator()() const { return false; }
};

template <typename VT>
struct Vec16;  // 16-byte vector of VT
template <>
struct Vec16<float> { using T = float4; static __device__ __forceinline__ float4 zero() { return make_float4(0.f, 0.f, 0.f, 0.f); } };
template <>
struct Vec16<double> { using T = double2; static __device__ __forceinline__ double2 zero() { return make_double2(0.0, 0.0); } };

// The product loop of one numeric row: CTA-per-row groups in flat mode use the block-level
// flattened loop; otherwise the per-sub-group loop plus the CTA pass over deferred long B rows.
template <int TPR, typename VT, typename BF, typename F>
__device__ __forceinline__ void num_products(const NumArgs& a, bool active, int row, int t, int long_len, int* s_list,
                                             int* s_lcnt, BF* bf, long long* ws, F&& f) {
  const VT* av = static_cast<const VT*>(a.a_val);
  const VT* bv = static_cast<const VT*>(a.b_val);
  if constexpr (TPR > 32) {
    if (a.flat) {
      for_each_product_block<true, false, VT, TPR>(a.a_rpt, a.a_col, av, a.b_rpt, a.b_col, bv, active, row, t, bf, ws,
                                                   f, NoStop{});
      return;
    }
  }
  if (active)
    products<true, false, VT, TPR>(a.flat, a.a_rpt, a.a_col, av, a.b_rpt, a.b_col, bv, row, t, TPR, a.vw_log2, f,
                                   NoStop{}, long_len, s_lcnt);
  if constexpr (TPR > 32) {
    if (long_len > 0)
      for_long_products<true, false, VT>(a.a_rpt, a.a_col, av, a.b_rpt, a.b_col, bv, active, row, t, TPR, long_len,
                                         s_list, s_lcnt, bf, f, NoStop{});
  }
}

// Scratch of the two-level bitmap rank (CTA-per-row groups).
struct Rank2 {
  unsigned* fine;    // [upper] bits of the non-empty 32-column blocks, compacted
  uint16_t* pre2;    // [upper] exclusive prefix popcount of fine (rank of the block's first key)
  unsigned* l1;      // [l1_words] level-1 bitmap: bit = 32-column block is non-empty
  unsigned* p1;      // [l1_words] exclusive prefix popcount of l1 (compact index of a block)
};

// Shared atomicOr of one key's bit (ATOMS.OR; a software peer reduction with a partial-warp
// __reduce_or_sync mask measured 3x slower than letting the atomic unit serialise same-word lanes).
__device__ __forceinline__ void or_aggregated(bool valid, unsigned* base, int idx, unsigned bits) {
  if (valid) atomicOr(base + idx, bits);
}

// (b)+(c) for CTA-per-row groups.  (b) gather: every thread takes its T/TPR contiguous slots into
// registers, the occupied ones are compacted to the front of the table (block scan; the table is
// no longer probed) and the row's column range [lo, hi] is reduced on the way.  (c) rank of every
// key = number of smaller keys of the row, from a two-level bitmap over [lo, hi]:
// level 1 marks the non-empty 32-column blocks (R/1024 words), its prefix popcount gives each
// non-empty block a compact index b, level 2 holds the 32-bit pattern of block b, and
// rank(key) = pre2[b] + popc(fine[b] & below(key)).  O(n + R/1024) work on the n compacted keys
// (KPT = upper/TPR per thread, kept in registers), no sorting, no crowding (a dense cluster only
// fills level-2 words).  Keys are distinct: the result is the unique ascending order.
template <typename VT, int TPR, int T, int KPT>
__device__ __forceinline__ long long gather_rank_2level(int* Kp, VT* Vp, const Rank2& r2, long long* ws, int* lohi,
                                                        bool active, int32_t* cc, VT* cv, long long cn) {
  constexpr int SPT = T / TPR;  // slots per thread, a multiple of 4
  static_assert(SPT % 4 == 0, "slots per thread");
  const int t = threadIdx.x;
  int ks[SPT];
  VT vs[SPT];
  int cnt = 0, mn = INT_MAX, mx = -1;
  {
    const int4* k4 = reinterpret_cast<const int4*>(Kp + t * SPT);
#pragma unroll
    for (int i = 0; i < SPT / 4; ++i) {
      const int4 kv = k4[i];
      ks[4 * i] = kv.x; ks[4 * i + 1] = kv.y; ks[4 * i + 2] = kv.z; ks[4 * i + 3] = kv.w;
    }
#pragma unroll
    for (int i = 0; i < SPT; ++i) {
      vs[i] = Vp[t * SPT + i];
      if (ks[i] >= 0) { ++cnt; mn = min(mn, ks[i]); mx = max(mx, ks[i]); }
    }
  }
  long long n;
  int off = (int)Grp<TPR>::excl_scan(cnt, &n, ws);  // its barriers order the reads before the writes
  Grp<TPR>::minmax(mn, mx, lohi);
#pragma unroll
  for (int i = 0; i < SPT; ++i)
    if (ks[i] >= 0) { Kp[off] = ks[i]; Vp[off] = vs[i]; ++off; }
  const int lo = lohi[0], hi = lohi[1];
  const int W1 = hi >= lo ? (int)(((unsigned)(hi - lo)) >> 10) + 1 : 0;
  for (int w = t; w < W1; w += TPR) r2.l1[w] = 0u;
  __syncthreads();
  int kk[KPT];
  unsigned dd[KPT];
#pragma unroll
  for (int m = 0; m < KPT; ++m) {
    const int j = t + m * TPR;
    kk[m] = j < n ? Kp[j] : -1;
    dd[m] = (unsigned)(kk[m] - lo);
    if (kk[m] >= 0) atomicOr(r2.l1 + (dd[m] >> 10), 1u << ((dd[m] >> 5) & 31));
  }
  __syncthreads();
  long long nb = 0;
  {
    const int per = (W1 + TPR - 1) / TPR;
    const int w0 = t * per, w1 = min(W1, w0 + per);
    long long loc = 0;
    for (int w = w0; w < w1; ++w) loc += __popc(r2.l1[w]);
    long long run = Grp<TPR>::excl_scan(loc, &nb, ws);
    for (int w = w0; w < w1; ++w) { r2.p1[w] = (unsigned)run; run += __popc(r2.l1[w]); }
  }
  for (int b = t; b < (int)nb; b += TPR) r2.fine[b] = 0u;
  __syncthreads();
  int bb[KPT];
#pragma unroll
  for (int m = 0; m < KPT; ++m) {
    if (kk[m] < 0) continue;
    const unsigned w = dd[m] >> 10, bit = (dd[m] >> 5) & 31;
    bb[m] = (int)(r2.p1[w] + __popc(r2.l1[w] & ((1u << bit) - 1u)));
    atomicOr(r2.fine + bb[m], 1u << (dd[m] & 31));
  }
  __syncthreads();
  long long n_total = 0;
  {
    const int per = (int)((nb + TPR - 1) / TPR);
    const int b0 = t * per, b1 = min((int)nb, b0 + per);
    long long loc = 0;
    for (int b = b0; b < b1; ++b) loc += __popc(r2.fine[b]);
    long long run = Grp<TPR>::excl_scan(loc, &n_total, ws);
    for (int b = b0; b < b1; ++b) { r2.pre2[b] = (uint16_t)run; run += __popc(r2.fine[b]); }
  }
  __syncthreads();
  if (active) {
#pragma unroll
    for (int m = 0; m < KPT; ++m) {
      if (kk[m] < 0) continue;
      const long long r = (long long)r2.pre2[bb[m]] + __popc(r2.fine[bb[m]] & ((1u << (dd[m] & 31)) - 1u));
      if (r < cn) { cc[r] = kk[m]; cv[r] = Vp[t + m * TPR]; }
    }
  }
  return n_total;
}

// One row: (0) init, (a) accumulate, (b) gather into buckets, (c) rank + write.
// Kp/Vp: the key/value tables (shared or global); Keys/Vals: their probe/add accessors.
template <typename VT, int TPR, bool GLOBAL, bool RANK2 = false, int TT = 0, int KPT = 0, typename Keys,
          typename Vals, typename SIdx, typename BF>
__device__ __forceinline__ void num_row(const NumArgs& a, bool active, int row, const Keys& K, const Vals& V,
                                        int* Kp, VT* Vp, int* Bc, SIdx* S, unsigned mask, int NB, int* lohi,
                                        long long* ws, int* s_list, int* s_lcnt, unsigned* wscr,
                                        BF* bf, const Rank2& r2 = Rank2{}) {
  const int t = Grp<TPR>::lane();
  const unsigned T = mask + 1;
  if (TPR > 32 && t == 0) *s_lcnt = 0;  // pass-1 "deferred a long row" flag (read after a barrier)
  if constexpr (!GLOBAL) {
    // Range-offset hash: when the row's column span R fits the table, slot =
    // key - lo_i (collision-free, order-preserving).  Vp[0..R) accumulates; the bytes of
    // Kp[0..R/4) flag occupancy (plain idempotent stores; structural zeros stay); the gather is
    // an in-order compaction of the flags.
    if (active && a.rlohi != nullptr) {
      const int2 rr = __ldg(a.rlohi + row);
      const long long R = (long long)rr.y - rr.x + 1;
      if (R > 0 && R <= (long long)T) {  // uniform within the row group
        const int lo = rr.x;
        const int long_len = TPR > 32 ? a.long_len : 0;
        const int vwl = a.vw_log2;
        const int ncopy = TPR >> vwl;  // one private accumulator row per sub-group
        const long long Rp = (R + 3) & ~3LL;
        const unsigned kb = smem_u32(Kp);
        const bool priv = a.priv_ok &&
                          ncopy * Rp * (long long)sizeof(VT) + Rp <= (long long)T * (long long)(sizeof(VT) + 4);
        long long n_total;
        const long long c0 = a.c_rpt[row];
        const long long cn = a.c_rpt[row + 1] - c0;
        VT* __restrict__ cv = static_cast<VT*>(a.c_val) + c0;
        int32_t* __restrict__ cc = a.c_col + c0;
        if (priv) {
          // Private accumulators: sub-group g adds into P[g][0..R) with plain read-modify-
          // writes (its lanes hold distinct columns of one B row; WSYNC reconverges it per A
          // non-zero), flags in the Rp bytes after the copies; the copies are summed in fixed
          // order at compaction time, so values are deterministic run to run.
          VT* P = Vp;
          unsigned char* fl = reinterpret_cast<unsigned char*>(P + ncopy * Rp);
          const unsigned fb = smem_u32(fl);
          using V16 = typename Vec16<VT>::T;
          constexpr int per = 16 / sizeof(VT);
          V16* v16 = reinterpret_cast<V16*>(P);
          for (long long s = t; s < ncopy * Rp / per; s += TPR) v16[s] = Vec16<VT>::zero();
          int4* f4 = reinterpret_cast<int4*>(fl);
          for (long long s = t; s < (Rp + 15) / 16; s += TPR) f4[s] = make_int4(0, 0, 0, 0);
          Grp<TPR>::sync();
          VT* __restrict__ mine = P + (t >> vwl) * Rp;
          auto f = [&](int key, VT prod) {
            const unsigned d = (unsigned)(key - lo);
            st_s8(fb + d, 1);
            mine[d] += prod;
          };
          for_each_product<true, false, VT, true>(a.a_rpt, a.a_col, static_cast<const VT*>(a.a_val), a.b_rpt,
                                                  a.b_col, static_cast<const VT*>(a.b_val), row, t, TPR, vwl, f,
                                                  NoStop{}, long_len, s_lcnt);
          if constexpr (TPR > 32) {
            if (long_len > 0)
              for_long_products<true, false, VT, true>(a.a_rpt, a.a_col, static_cast<const VT*>(a.a_val), a.b_rpt,
                                                       a.b_col, static_cast<const VT*>(a.b_val), true, row, t, TPR,
                                                       long_len, s_list, s_lcnt, bf, f, NoStop{});
          }
          Grp<TPR>::sync();
          const int words = (int)(Rp >> 2);
          const int pw = (words + TPR - 1) / TPR;
          const int w0 = t * pw, w1 = min(words, w0 + pw);
          const unsigned* fw = reinterpret_cast<const unsigned*>(fl);
          long long loc = 0;
          for (int w = w0; w < w1; ++w) loc += __popc(fw[w]);
          long long r = Grp<TPR>::excl_scan(loc, &n_total, ws);
          if (t == 0 && cn != n_total) atomicOr(a.err_flags, 2);
          for (int w = w0; w < w1; ++w) {
            unsigned bits = fw[w];
            while (bits) {
              const int d = w * 4 + ((__ffs(bits) - 1) >> 3);
              bits &= bits - 1;
              VT v = P[d];
              for (int c = 1; c < ncopy; ++c) v += P[c * Rp + d];
              if (r < cn) { cc[r] = lo + d; cv[r] = v; }
              ++r;
            }
          }
          Grp<TPR>::sync();
          return;
        }
        const int words = (int)((R + 3) >> 2);  // 4 flag bytes per word
        using V16 = typename Vec16<VT>::T;
        constexpr int per = 16 / sizeof(VT);
        V16* v16 = reinterpret_cast<V16*>(Vp);
        for (int s = t; s < (int)((R + per - 1) / per); s += TPR) v16[s] = Vec16<VT>::zero();
        int4* k4 = reinterpret_cast<int4*>(Kp);
        for (int s = t; s < (words + 3) / 4; s += TPR) k4[s] = make_int4(0, 0, 0, 0);
        Grp<TPR>::sync();
        auto f = [&](int key, VT prod) {
          const unsigned d = (unsigned)(key - lo);
          st_s8(kb + d, 1);
          V.add(d, prod);
        };
        num_products<TPR, VT>(a, true, row, t, long_len, s_list, s_lcnt, bf, ws, f);
        Grp<TPR>::sync();
        // in-order compaction: thread owns a contiguous run of flag words
        const int pw = (words + TPR - 1) / TPR;
        const int w0 = t * pw, w1 = min(words, w0 + pw);
        long long loc = 0;
        for (int w = w0; w < w1; ++w) loc += __popc((unsigned)Kp[w]);
        long long r = Grp<TPR>::excl_scan(loc, &n_total, ws);
        if (t == 0 && cn != n_total) atomicOr(a.err_flags, 2);
        for (int w = w0; w < w1; ++w) {
          unsigned bits = (unsigned)Kp[w];
          while (bits) {
            const int d = w * 4 + ((__ffs(bits) - 1) >> 3);
            bits &= bits - 1;
            if (r < cn) { cc[r] = lo + d; cv[r] = Vp[d]; }
            ++r;
          }
        }
        Grp<TPR>::sync();
        return;
      }
    }
  }
  // (0) keys <- -1 (Alg. 5 precondition), values <- 0; 16-byte stores
  {
    int4* k4 = reinterpret_cast<int4*>(Kp);
    for (unsigned s = t; s < T / 4; s += TPR) k4[s] = make_int4(-1, -1, -1, -1);
    using V16 = typename Vec16<VT>::T;
    V16* v16 = reinterpret_cast<V16*>(Vp);
    constexpr unsigned per = 16 / sizeof(VT);
    for (unsigned s = t; s < T / per; s += TPR) v16[s] = Vec16<VT>::zero();
  }
  Grp<TPR>::sync();

  // (a) accumulate
  {
    auto f = [&](int key, VT prod) {  // prod = a_ik * b_kj (Alg. 1 "value")
      bool ins;
      const unsigned s = probe(K, mask, key, ins);
      V.add(s, prod);
    };
    const int long_len = TPR > 32 ? a.long_len : 0;
    num_products<TPR, VT>(a, active, row, t, long_len, s_list, s_lcnt, bf, ws, f);
  }
  Grp<TPR>::sync();
  if constexpr (RANK2) {
    if (a.prof && threadIdx.x == 0) a.prof[4 * blockIdx.x + 2] = gtimer();
    const long long c0 = active ? a.c_rpt[row] : 0;
    const long long cn = active ? a.c_rpt[row + 1] - c0 : 0;
    const long long n_total = gather_rank_2level<VT, TPR, TT, KPT>(Kp, Vp, r2, ws, lohi, active, a.c_col + c0,
                                                                   static_cast<VT*>(a.c_val) + c0, cn);
    if (t == 0 && active && cn != n_total) atomicOr(a.err_flags, 2);
    Grp<TPR>::sync();
    if (a.prof && threadIdx.x == 0) {
      unsigned smid;
      asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
      a.prof[4 * blockIdx.x + 3] = gtimer();
      a.prof[4 * blockIdx.x + 0] = ((unsigned long long)smid << 32) | (unsigned)row;
    }
    return;
  }

  // (b) gather: column range [lo, hi] of the row (group min/max over the table)
  const int4* k4 = reinterpret_cast<const int4*>(Kp);
  {
    int mn = INT_MAX, mx = -1;
    for (unsigned s4 = t; s4 < T / 4; s4 += TPR) {
      const int4 kv = k4[s4];
      mx = max(max(mx, kv.x), max(kv.y, max(kv.z, kv.w)));
      mn = min(mn, kv.x < 0 ? INT_MAX : kv.x);
      mn = min(mn, kv.y < 0 ? INT_MAX : kv.y);
      mn = min(mn, kv.z < 0 ? INT_MAX : kv.z);
      mn = min(mn, kv.w < 0 ? INT_MAX : kv.w);
    }
    Grp<TPR>::minmax(mn, mx, lohi);
  }
  const int lo = lohi[0], hi = lohi[1];
  const long long c0 = active ? a.c_rpt[row] : 0;
  const long long cn = active ? a.c_rpt[row + 1] - c0 : 0;
  VT* __restrict__ cv = static_cast<VT*>(a.c_val) + c0;
  int32_t* __restrict__ cc = a.c_col + c0;
  long long n_total = 0;
  if constexpr (GLOBAL) {
    // (c) global-memory rows: bitmap rank over [lo, hi]; rank(key) = #set bits below it
    // (prefix popcount per 32-bit word + popc of the partial word).  Bc = bitmap, S = prefix.
    const int W = hi >= lo ? (int)(((unsigned)(hi - lo)) >> 5) + 1 : 0;
    unsigned* bits = reinterpret_cast<unsigned*>(Bc);
    for (int w = t; w < W; w += TPR) bits[w] = 0u;
    Grp<TPR>::sync();
    for (unsigned s4 = t; s4 < T / 4; s4 += TPR) {
      const int4 kv = k4[s4];
      if (kv.x >= 0) atomicOr(bits + ((kv.x - lo) >> 5), 1u << ((kv.x - lo) & 31));
      if (kv.y >= 0) atomicOr(bits + ((kv.y - lo) >> 5), 1u << ((kv.y - lo) & 31));
      if (kv.z >= 0) atomicOr(bits + ((kv.z - lo) >> 5), 1u << ((kv.z - lo) & 31));
      if (kv.w >= 0) atomicOr(bits + ((kv.w - lo) >> 5), 1u << ((kv.w - lo) & 31));
    }
    Grp<TPR>::sync();
    {
      const int per = (W + TPR - 1) / TPR;
      const int w0 = t * per, w1 = min(W, w0 + per);
      long long loc = 0;
      for (int w = w0; w < w1; ++w) loc += __popc(bits[w]);
      long long run = Grp<TPR>::excl_scan(loc, &n_total, ws);
      for (int w = w0; w < w1; ++w) { S[w] = (SIdx)run; run += __popc(bits[w]); }
    }
    Grp<TPR>::sync();
    if (active) {
      if (t == 0 && cn != n_total) atomicOr(a.err_flags, 2);
      for (unsigned s = t; s < T; s += TPR) {
        const int key = Kp[s];
        if (key < 0) continue;
        const unsigned d = (unsigned)(key - lo);
        const int r = (int)S[d >> 5] + __popc(bits[d >> 5] & ((1u << (d & 31)) - 1u));
        if (r < cn) { cc[r] = key; cv[r] = Vp[s]; }
      }
    }
  } else {
    int shift = 0, nb = 0;
    if (hi >= lo) {
      const unsigned R = (unsigned)(hi - lo);
      while ((R >> shift) >= (unsigned)NB) ++shift;
      nb = (int)(R >> shift) + 1;
    }
    if (shift <= 2 || TPR > 32) {
      // Buckets of width 2^shift over [lo, hi]: histogram, exclusive scan, scatter of the
      // slot indices into bucket order (Bc[b] = start of bucket b afterwards).
      for (int b = t; b <= nb; b += TPR) Bc[b] = 0;
      Grp<TPR>::sync();
      for (unsigned s4 = t; s4 < T / 4; s4 += TPR) {
        const int4 kv = k4[s4];
        if (kv.x >= 0) atomicAdd(&Bc[1 + ((kv.x - lo) >> shift)], 1);
        if (kv.y >= 0) atomicAdd(&Bc[1 + ((kv.y - lo) >> shift)], 1);
        if (kv.z >= 0) atomicAdd(&Bc[1 + ((kv.z - lo) >> shift)], 1);
        if (kv.w >= 0) atomicAdd(&Bc[1 + ((kv.w - lo) >> shift)], 1);
      }
      Grp<TPR>::sync();
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
      for (unsigned s4 = t; s4 < T / 4; s4 += TPR) {
        const int4 kv = k4[s4];
        const unsigned s = 4 * s4;
        if (kv.x >= 0) S[atomicAdd(&Bc[1 + ((kv.x - lo) >> shift)], 1)] = (SIdx)(s);
        if (kv.y >= 0) S[atomicAdd(&Bc[1 + ((kv.y - lo) >> shift)], 1)] = (SIdx)(s + 1);
        if (kv.z >= 0) S[atomicAdd(&Bc[1 + ((kv.z - lo) >> shift)], 1)] = (SIdx)(s + 2);
        if (kv.w >= 0) S[atomicAdd(&Bc[1 + ((kv.w - lo) >> shift)], 1)] = (SIdx)(s + 3);
      }
      Grp<TPR>::sync();
      if (t == 0 && active && cn != n_total) atomicOr(a.err_flags, 2);
      // (c1) thread per key: rank = bucket start + #smaller keys in its bucket, for buckets of at
      // most kSparseBucket keys (every bucket when shift <= 2: width <= 4)
      constexpr int kSparseBucket = 8;
      if (active) {
        for (int p = t; p < (int)n_total; p += TPR) {
          const unsigned s = S[p];
          const int key = Kp[s];
          const int b = (key - lo) >> shift;
          const int st = Bc[b], en = Bc[b + 1];
          if (TPR > 32 && en - st > kSparseBucket) continue;  // crowded: (c4) below
          int r = st;
          for (int q = st; q < en; ++q) r += (Kp[S[q]] < key);
          if (r < cn) { cc[r] = key; cv[r] = Vp[s]; }
        }
      }
      if constexpr (TPR > 32) {
        // (c4) crowded buckets, one warp each: the warp scans 32 bucket counts at a time and
        // visits only the crowded ones (sparse wide rows — graph shapes — have ~1 key per
        // bucket and no warp work here).  <= 32 keys -> rank by shuffle comparisons; denser
        // buckets of width <= 32 * kWarpBitmapWords -> per-warp bitmap + popcount prefix; wider
        // -> comparisons.
        constexpr int MW = kWarpBitmapWords<TPR>;  // bitmap words per warp
        constexpr int WPL = MW / 32;
        const int wid = t >> 5, ln = t & 31;
        unsigned* wb = wscr + wid * 2 * MW;
        unsigned* wp = wb + MW;
        const int words = (int)(((1u << shift) + 31) >> 5);
        // bucket b belongs to warp b % NW (crowded buckets are usually adjacent — the dense
        // part of a row's column range — so a round-robin split balances them over the warps)
        constexpr int NW = TPR / 32;
        for (int k0 = 0; active && wid + k0 * NW < nb; k0 += 32) {
          const int bl = wid + (k0 + ln) * NW;
          const int cl = bl < nb ? Bc[bl + 1] - Bc[bl] : 0;
          unsigned crowd = __ballot_sync(0xffffffffu, cl > kSparseBucket);
          while (crowd) {
            const int b = wid + (k0 + __ffs(crowd) - 1) * NW;
            crowd &= crowd - 1;
            const int st = Bc[b], en = Bc[b + 1], c = en - st;  // warp-uniform
            const int base = lo + (b << shift);
            if (c <= 32) {
              const unsigned slot = ln < c ? (unsigned)S[st + ln] : 0u;
              const int key = ln < c ? Kp[slot] : INT_MAX;
              int r = 0;
              for (int m = 0; m < c; ++m) r += __shfl_sync(0xffffffffu, key, m) < key;
              if (ln < c && st + r < cn) { cc[st + r] = key; cv[st + r] = Vp[slot]; }
            } else if (words <= MW) {
              for (int w = ln; w < words; w += 32) wb[w] = 0u;
              __syncwarp();
              for (int p = st + ln; p < en; p += 32) {
                const unsigned d = (unsigned)(Kp[S[p]] - base);
                atomicOr(wb + (d >> 5), 1u << (d & 31));
              }
              __syncwarp();
              unsigned loc[WPL], sum = 0;
#pragma unroll
              for (int u = 0; u < WPL; ++u) {
                loc[u] = ln * WPL + u < words ? __popc(wb[ln * WPL + u]) : 0u;
                sum += loc[u];
              }
              unsigned incl = sum;
#pragma unroll
              for (int o = 1; o < 32; o <<= 1) {
                const unsigned y = __shfl_up_sync(0xffffffffu, incl, o);
                if (ln >= o) incl += y;
              }
              unsigned ex = incl - sum;
#pragma unroll
              for (int u = 0; u < WPL; ++u) { wp[ln * WPL + u] = ex; ex += loc[u]; }
              __syncwarp();
              for (int p = st + ln; p < en; p += 32) {
                const unsigned slot = S[p];
                const int key = Kp[slot];
                const unsigned d = (unsigned)(key - base);
                const int r = st + (int)wp[d >> 5] + __popc(wb[d >> 5] & ((1u << (d & 31)) - 1u));
                if (r < cn) { cc[r] = key; cv[r] = Vp[slot]; }
              }
              __syncwarp();
            } else {
              for (int p = st + ln; p < en; p += 32) {
                const unsigned slot = S[p];
                const int key = Kp[slot];
                int r = st;
                for (int q = st; q < en; ++q) r += (Kp[S[q]] < key);
                if (r < cn) { cc[r] = key; cv[r] = Vp[slot]; }
              }
            }
          }
        }
      }
    } else {
      // (c2) wide, clustered ranges: compact the slot indices, bitonic-sort them by key in
      // shared memory (n' = next_pow2(n) <= the group's nnz bound), write C coalesced.
      int* cnt = Bc;
      if (t == 0) *cnt = 0;
      Grp<TPR>::sync();
      for (unsigned s = t; s < T; s += TPR) {
        const bool occ = Kp[s] >= 0;
        const unsigned bal = __ballot_sync(Grp<TPR>::mask(), occ);
        if (bal) {  // uniform across the row group
          const int lead = __ffs(bal) - 1;
          int base = 0;
          if ((threadIdx.x & 31) == lead) base = atomicAdd(cnt, __popc(bal));
          base = __shfl_sync(Grp<TPR>::mask(), base, lead);
          if (occ) S[base + __popc(bal & ((1u << (threadIdx.x & 31)) - 1u))] = (SIdx)s;
        }
      }
      Grp<TPR>::sync();
      const int n = *cnt;
      n_total = n;
      int np2 = 1;
      while (np2 < n) np2 <<= 1;
      constexpr SIdx kSent = (SIdx)~SIdx(0);
      for (int p = n + t; p < np2; p += TPR) S[p] = kSent;
      Grp<TPR>::sync();
      auto keyof = [&](SIdx x) { return x == kSent ? INT_MAX : Kp[x]; };
      for (int k = 2; k <= np2; k <<= 1) {
        for (int j = k >> 1; j > 0; j >>= 1) {
          for (int q = t; q < (np2 >> 1); q += TPR) {
            const int i = ((q & ~(j - 1)) << 1) | (q & (j - 1));
            const int l = i | j;
            const SIdx x = S[i], y = S[l];
            const bool up = (i & k) == 0;
            if ((keyof(x) > keyof(y)) == up) { S[i] = y; S[l] = x; }
          }
          Grp<TPR>::sync();
        }
      }
      if (active) {
        if (t == 0 && cn != n_total) atomicOr(a.err_flags, 2);
        for (int p = t; p < n && p < cn; p += TPR) {
          const unsigned s = S[p];
          cc[p] = Kp[s];
          cv[p] = Vp[s];
        }
      }
    }
  }
  Grp<TPR>::sync();
}

template <typename VT, int T, int TPR, int BS, long long UPPER, bool RANK2>
__global__ __launch_bounds__(BS, (RANK2 && BS >= 512) ? 2048 / BS : 1) void k_num_smem(NumArgs a) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  __shared__ long long ws[33];
  constexpr int RPB = BS / TPR;
  __shared__ int s_lohi[2 * RPB];
  __shared__ int s_list[TPR > 32 ? kLongChunk : 1], s_lcnt;
  // per-warp bucket bitmap+prefix of the (c4) sort, aliased with the block-flat product scratch
  // (used in different phases of a row; separated by barriers)
  constexpr int kWscrBytes = TPR > 32 ? (TPR / 32) * 8 * kWarpBitmapWords<TPR> : 4;
  // two-level rank: the product-loop chunk (one chunk of <= TPR A non-zeros) lives in the rank
  // scratch (fine/pre2, unused until the gather), so the static shared memory stays small
  using BF = BlockFlat<VT, RANK2 ? flat_chunk_of<TPR>() : kFlatChunk>;
  static_assert(!RANK2 || sizeof(BF) <= (size_t)UPPER * 6, "chunk must fit the rank scratch");
  constexpr int kAuxBytes = (TPR > 32 && !RANK2) ? (kWscrBytes > (int)sizeof(BF) ? kWscrBytes : (int)sizeof(BF)) : 16;
  __shared__ __align__(16) unsigned char s_aux[kAuxBytes];
  unsigned* s_wscr = reinterpret_cast<unsigned*>(s_aux);
  constexpr int NB = num_nbuckets(T);
  constexpr int RB = num_row_bytes<VT>(T, UPPER);
  const int g = threadIdx.x / TPR;
  unsigned char* base = smem_raw + g * RB;
  VT* Vp = reinterpret_cast<VT*>(base);
  int* Kp = reinterpret_cast<int*>(base + T * sizeof(VT));
  int* Bc = Kp + T;
  uint16_t* S = reinterpret_cast<uint16_t*>(Bc + NB + 1);
  const long long ridx = (long long)blockIdx.x * RPB + g;
  const bool active = ridx < a.nrows;
  const int row = active ? a.rows[ridx] : 0;
  if constexpr (RANK2) {
    static_assert(TPR == BS, "two-level rank: one row per CTA");
    if (a.prof && threadIdx.x == 0) a.prof[4 * blockIdx.x + 1] = gtimer();
    Rank2 r2;
    r2.fine = reinterpret_cast<unsigned*>(Kp + T);
    r2.pre2 = reinterpret_cast<uint16_t*>(r2.fine + UPPER);
    r2.l1 = reinterpret_cast<unsigned*>(smem_raw + align16(T * (int)sizeof(VT) + T * 4 + (int)UPPER * 6));
    r2.p1 = r2.l1 + a.l1_words;
    num_row<VT, TPR, false, true, T, (int)(UPPER / TPR)>(a, active, row, SKeys{smem_u32(Kp)}, SVals<VT>{smem_u32(Vp)}, Kp, Vp,
                                  reinterpret_cast<int*>(r2.fine), (uint16_t*)nullptr, T - 1, NB, s_lohi, ws, s_list,
                                  &s_lcnt, s_wscr, reinterpret_cast<BF*>(r2.fine), r2);
  } else {
    num_row<VT, TPR, false>(a, active, row, SKeys{smem_u32(Kp)}, SVals<VT>{smem_u32(Vp)}, Kp, Vp, Bc, S, T - 1, NB,
                            s_lohi + 2 * g, ws, s_list, &s_lcnt, s_wscr, reinterpret_cast<BF*>(s_aux));
  }
}

template <typename VT>
__global__ __launch_bounds__(1024) void k_num_global(NumArgs a) {
  __shared__ long long ws[33];
  __shared__ int s_lohi[2];
  __shared__ BlockFlat<VT> s_bf;
  __shared__ int s_list[kLongChunk], s_lcnt;
  unsigned char* slab = static_cast<unsigned char*>(a.slab) + (long long)blockIdx.x * a.slab_stride;
  VT* Vp = reinterpret_cast<VT*>(slab);
  int* Kp = reinterpret_cast<int*>(Vp + a.slab_T);
  int* Bc = Kp + a.slab_T;              // bitmap over [lo, hi]: bitmap_words ints
  int* S = Bc + a.bitmap_words;         // prefix popcount per bitmap word
  for (long long i = blockIdx.x; i < a.nrows; i += gridDim.x) {
    const int row = a.rows[i];
    const long long n = a.c_rpt[row + 1] - a.c_rpt[row];
    long long T = 64;
    while (T < 2 * n) T <<= 1;
    if (T > a.slab_T) T = a.slab_T;
    num_row<VT, 1024, true>(a, true, row, GKeys{Kp}, GVals<VT>{Vp}, Kp, Vp, Bc, S, (unsigned)(T - 1), 0,
                            s_lohi, ws, s_list, &s_lcnt, nullptr, &s_bf);
  }
}

template <typename VT, int T, int TPR, int BS, long long UPPER, bool RANK2>
cudaError_t launch_num_k(cudaStream_t s, const NumArgs& a, int smem) {
  static PerDevice configured;
  auto& cfg = configured.here();
  if (smem > cfg.load()) {
    cudaError_t e = cudaFuncSetAttribute(k_num_smem<VT, T, TPR, BS, UPPER, RANK2>,
                                         cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    if (e != cudaSuccess) return e;
    cfg.store(smem);
  }
  NumArgs b = a;
  const int max_vw = TPR < 32 ? TPR : 32;
  while ((1 << b.vw_log2) > max_vw) --b.vw_log2;
  constexpr int RPB = BS / TPR;
  const long long grid = (a.nrows + RPB - 1) / RPB;
  k_num_smem<VT, T, TPR, BS, UPPER, RANK2><<<(unsigned)grid, BS, smem, s>>>(b);
  return cudaGetLastError();
}

// static shared memory of k_num_smem besides the dynamic tables
template <typename VT, int TPR>
constexpr int num_static_bytes() {  // k_num_smem<..., RANK2 = true>
  return 33 * 8 + 8 * 32 + 4 * kLongChunk + 16 + 16;
}

template <typename VT, int T, int TPR, int BS, long long UPPER>
cudaError_t launch_num_old(cudaStream_t s, const NumArgs& a);

template <typename VT, int T, int TPR, int BS, long long UPPER>
cudaError_t launch_num(cudaStream_t s, const NumArgs& a) {
  if constexpr (TPR > 32) {  // CTA per row: two-level bitmap rank when its scratch fits
    const long long smem2 = num_cta_bytes<VT>(T, UPPER, a.l1_words);
    if (a.l1_words > 0 && smem2 + num_static_bytes<VT, TPR>() <= kSmemLimit)
      return launch_num_k<VT, T, TPR, BS, UPPER, true>(s, a, (int)smem2);
  }
  return launch_num_old<VT, T, TPR, BS, UPPER>(s, a);
}

template <typename VT, int T, int TPR, int BS, long long UPPER>
cudaError_t launch_num_old(cudaStream_t s, const NumArgs& a) {
  constexpr int RPB = BS / TPR;
  constexpr int smem = RPB * num_row_bytes<VT>(T, UPPER);
  static_assert(smem + 33 * 8 + 8 * RPB + 4 * kLongChunk + 16 +
                    (TPR > 32 ? (TPR / 32 * 8 * kWarpBitmapWords<TPR> > (int)sizeof(BlockFlat<VT>)
                                     ? TPR / 32 * 8 * kWarpBitmapWords<TPR>
                                     : (int)sizeof(BlockFlat<VT>)) : 4) <= kSmemLimit,
                "numeric table too large");
  return launch_num_k<VT, T, TPR, BS, UPPER, false>(s, a, smem);
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
