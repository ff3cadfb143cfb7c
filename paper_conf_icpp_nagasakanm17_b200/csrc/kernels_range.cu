// kernels_range.cu — warp-per-row kernels for "range rows" (B200 addition).
//
// A range row is a row of C whose exact column span R_i = hi_i - lo_i + 1 (computed with n_prod
// in step (1), k_nprod_group) is narrow (R_i <= kRangeMaxSpan, R_i <= 4 n_prod_i) and whose
// n_prod_i is large enough to feed a warp — the rows of FEM / banded / stencil matrices (all of
// the cant-like config).  For them the hash of Alg. 5 degenerates to the
// collision-free, order-preserving offset hash h = key - lo_i over a table of R_i slots, and one
// warp owns the whole row:
//
//   * product walk (Alg. 3/4, flattened): the row's A non-zeros are taken 32 at
//     a time; lane j loads the metadata of non-zero j (col_A, val_A, rpt_B pair) and the warp
//     scans the B-row lengths into a per-warp shared table, then the warp strides its 32 lanes
//     over the batch's concatenated products — every lane busy whatever the B-row lengths (the
//     lane-per-B-entry loop of Alg. 4 idles ~40% of the lanes on cant's 50-78-entry B rows);
//   * symbolic (step 3): byte flag[key - lo] = 1 (idempotent plain stores, no atomics); nnz_i =
//     number of set flags; the flags are also packed into a bitmap of the row's pattern in global
//     memory (R_i / 8 bytes per row), which the numeric kernel uses for the gather;
//   * numeric (step 7a): acc[c][key - lo] += a_ik * b_kj with a plain shared-memory read-modify-
//     write (sm_100a lowers shared float atomics to CAS loops).  B rows are strictly increasing
//     (checked by k_brow_minmax, else these rows take the hash groups), so lanes working on one B
//     row hold distinct columns; a 32-product step covers at most two B rows when they all have
//     >= 32 entries, and those two go to the two accumulator copies c = e & 1; otherwise the
//     step's B rows are applied one after another.  Values are deterministic run to run;
//   * gather + sort (7b/7c): the table is already in column order — the warp
//     walks the symbolic bitmap 32 columns at a time (popc prefix) and writes C coalesced.
//
// Scheduling: a persistent grid of one CTA per SM (up to 32 warps); CTA b owns a contiguous
// slice of the group's rows (the permutation keeps rows of a group in near-ascending order) and
// its warps take the slice's rows through a shared counter, so the rows in flight on one SM are
// neighbours and share most of their B rows — B is served from that SM's L1 (measured hit rate
// 93-98% on cant, vs 36% for the CTA-per-row groups).  Per-warp tables are R_cap (= max R_i of
// the group) slots, so shared memory does not limit occupancy the way the n_prod-sized tables of
// Table I do.
#include <cstdlib>

#include "spgemm_internal.cuh"

namespace spg {

namespace {

template <typename VT>
struct RVec;
template <>
struct RVec<float> {
  static __device__ __forceinline__ float ld(unsigned a) {
    float v;
    asm volatile("ld.shared.f32 %0, [%1];" : "=f"(v) : "r"(a));
    return v;
  }
  static __device__ __forceinline__ void st(unsigned a, float v) { asm volatile("st.shared.f32 [%0], %1;" ::"r"(a), "f"(v)); }
};
template <>
struct RVec<double> {
  static __device__ __forceinline__ double ld(unsigned a) {
    double v;
    asm volatile("ld.shared.f64 %0, [%1];" : "=d"(v) : "r"(a));
    return v;
  }
  static __device__ __forceinline__ void st(unsigned a, double v) { asm volatile("st.shared.f64 [%0], %1;" ::"r"(a), "d"(v)); }
};

// Per-warp metadata of one batch of 32 A non-zeros: product p of the batch (0 <= p < total)
// with end[e-1] <= p < end[e] is b_col[base[e] + p] (base = rpt_B[col_A] - start of e; 32-bit:
// range rows require rpt_B[k] < 2^31), scaled by av[e] = a_ik.  16 bytes per entry (one LDS.128).
constexpr int kMetaBatch = 32;
template <typename VT>
struct alignas(16) REnt {
  int base, end;
  VT av;
};
template <typename VT>
struct RMetaW {
  REnt<VT> e[kMetaBatch];
};
static_assert(sizeof(REnt<float>) == 16 && sizeof(REnt<double>) == 16 && sizeof(REnt<int>) == 16, "entry size");

__device__ __forceinline__ void st_u8(unsigned a) {  // flag byte = 1
  asm volatile("st.shared.u8 [%0], %1;" ::"r"(a), "h"((unsigned short)1));
}

template <typename VT>
__device__ __forceinline__ REnt<VT> lds_ent(unsigned a) {
  int4 v;
  asm volatile("ld.shared.v4.b32 {%0, %1, %2, %3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "r"(a));
  REnt<VT> r;
  r.base = v.x;
  r.end = v.y;
  if constexpr (sizeof(VT) == 8) r.av = __hiloint2double(v.w, v.z);
  else r.av = __int_as_float(v.z);
  return r;
}

// Row index source of the persistent grid: CTA b owns rows [c0, c1) of the group's slice; its
// warps take them in order through a shared counter (lane 0 increments, broadcast).
struct RowQueue {
  long long c0, c1;
  int* next;
  __device__ __forceinline__ long long pop(int lane) const {
    int i = 0;
    if (lane == 0) i = atomicAdd(next, 1);
    i = __shfl_sync(0xffffffffu, i, 0);
    const long long r = c0 + i;
    return r < c1 ? r : -1;
  }
};

__device__ __forceinline__ RowQueue row_queue(long long nrows, int* s_next) {
  if (threadIdx.x == 0) *s_next = 0;
  __syncthreads();
  const long long chunk = (nrows + gridDim.x - 1) / gridDim.x;
  const long long c0 = (long long)blockIdx.x * chunk;
  return RowQueue{c0, c0 + chunk < nrows ? c0 + chunk : nrows, s_next};
}

// Walk the products of one row (see the header).  step(valid, key, a_ik, b_kj, e, serial) is
// called once per 32-product step by every lane (e: the lane's A non-zero within the batch).
// `serial` (warp-uniform) is true when some B row of the batch has fewer than 32 entries: a step
// may then span more than two B rows (the numeric caller applies them one at a time).  Otherwise
// every lane crosses at most one B-row boundary per step, and its current B row (base, end,
// a_ik) stays in registers, refreshed from the per-warp table only when it crosses; two steps
// per iteration keep two gathers (four in numeric) in flight per lane.
template <bool NUM, typename VT, typename F>
__device__ __forceinline__ void range_products(const int64_t* __restrict__ a_rpt, const int32_t* __restrict__ a_col,
                                               const VT* __restrict__ a_val, const int64_t* __restrict__ b_rpt,
                                               const int32_t* __restrict__ b_col, const VT* __restrict__ b_val,
                                               int row, int lane, RMetaW<VT>* meta, F&& step) {
  const long long a0 = __ldg(a_rpt + row);
  const int na = (int)(__ldg(a_rpt + row + 1) - a0);
  const int32_t* __restrict__ ac = opaque(a_col + a0);
  const VT* __restrict__ avp = NUM ? opaque(a_val + a0) : nullptr;
  const REnt<VT>* __restrict__ ment = meta->e;
  const unsigned mb = smem_u32(meta->e);
  const int32_t* __restrict__ bc = opaque(b_col);
  const VT* __restrict__ bvp = NUM ? opaque(b_val) : nullptr;
  for (int bb = 0; bb < na; bb += kMetaBatch) {
    const int j = bb + lane;
    int b0 = 0, len = 0;
    VT av = VT(0);
    if (j < na) {
      const int kk = __ldg(ac + j);
      if (NUM) av = __ldg(avp + j);
      b0 = (int)__ldg(b_rpt + kk);
      len = (int)__ldg(b_rpt + kk + 1) - b0;
    }
    int incl = len;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
      const int y = __shfl_up_sync(0xffffffffu, incl, d);
      if (lane >= d) incl += y;
    }
    const int total = __shfl_sync(0xffffffffu, incl, 31);
    const bool serial = __any_sync(0xffffffffu, j < na && len < 32);
    {
      REnt<VT> en;
      en.base = b0 - (incl - len);
      en.end = incl;
      en.av = av;
      meta->e[lane] = en;
    }
    __syncwarp();
    if (!serial) {
      int e = 0;
      unsigned mp = mb;
      REnt<VT> cur = lds_ent<VT>(mp);
#pragma unroll 1
      for (int p0 = 0; p0 < total; p0 += 64) {  // warp-uniform trip count
        const int pa = p0 + lane, pb = pa + 32;
        const bool va = pa < total, vb = pb < total;
        if (va && pa >= cur.end) {  // crossed into the next B row (at most once per step)
          ++e;
          mp += 16u;
          cur = lds_ent<VT>(mp);
        }
        const int ea = e;
        const VT xa = cur.av;
        int ka = 0;
        VT wa = VT(0);
        if (va) {
          const unsigned q = (unsigned)(cur.base + pa);
          ka = __ldg(bc + q);
          if (NUM) wa = __ldg(bvp + q);
        }
        if (vb && pb >= cur.end) {
          ++e;
          mp += 16u;
          cur = lds_ent<VT>(mp);
        }
        int kb = 0;
        VT wb = VT(0);
        if (vb) {
          const unsigned q = (unsigned)(cur.base + pb);
          kb = __ldg(bc + q);
          if (NUM) wb = __ldg(bvp + q);
        }
        step(va, ka, xa, wa, ea, false);
        step(vb, kb, cur.av, wb, e, false);
      }
    } else {
      int e = 0;
#pragma unroll 1
      for (int p0 = 0; p0 < total; p0 += 32) {
        const int p = p0 + lane;
        const bool valid = p < total;
        if (valid)
          while (ment[e].end <= p) ++e;  // skips empty B rows
        int key = 0;
        VT w = VT(0);
        if (valid) {
          const unsigned q = (unsigned)(ment[e].base + p);
          key = __ldg(bc + q);
          if (NUM) w = __ldg(bvp + q);
        }
        step(valid, key, NUM ? ment[e].av : VT(0), w, e, true);
      }
    }
    __syncwarp();
  }
}

// Step (3) on range rows: per warp RMetaW | flags[rcap] bytes.  Writes nnz_i and the row's
// pattern bitmap (rwcap words per row, row r of the group's slice).
__global__ __launch_bounds__(1024, 1) void k_sym_range(SymArgs a, int rcap) {
  extern __shared__ __align__(16) unsigned char rsm[];
  __shared__ int s_next;
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  constexpr int kMetaBytes = (int)sizeof(RMetaW<int>);
  unsigned char* wb = rsm + (size_t)w * (kMetaBytes + rcap);
  RMetaW<int>* meta = reinterpret_cast<RMetaW<int>*>(wb);
  unsigned char* fl = wb + kMetaBytes;
  const unsigned fb = smem_u32(fl);
  const RowQueue rq = row_queue(a.nrows, &s_next);
  for (long long r = rq.pop(lane); r >= 0; r = rq.pop(lane)) {
    const int row = a.rows[r];
    const int2 rr = __ldg(a.rlohi + row);
    const int lo = rr.x, R = rr.y - rr.x + 1;  // 1 <= R <= rcap (group criterion)
    int4* f4 = reinterpret_cast<int4*>(fl);
    const int n16 = (R + 15) >> 4;
    for (int s = lane; s < n16; s += 32) f4[s] = make_int4(0, 0, 0, 0);
    __syncwarp();
    const unsigned fbl = opaque(fb - (unsigned)lo);  // flag of key = fbl + key
    range_products<false, int>(a.a_rpt, a.a_col, nullptr, a.b_rpt, a.b_col, nullptr, row, lane, meta,
                               [&](bool valid, int key, int, int, int, bool) {
                                 if (valid) st_u8(fbl + (unsigned)key);
                               });
    // pattern bitmap: lane packs the 32 flag bytes of word wd (0/1 bytes -> bits)
    int cnt = 0;
    unsigned* bits = a.rbits ? a.rbits + r * a.rwcap : nullptr;
    const int nw = (R + 31) >> 5;
    for (int wd = lane; wd < nw; wd += 32) {
      const int4* src = reinterpret_cast<const int4*>(fl + wd * 32);
      const int4 u = src[0], v = src[1];
      const unsigned x[8] = {(unsigned)u.x, (unsigned)u.y, (unsigned)u.z, (unsigned)u.w,
                             (unsigned)v.x, (unsigned)v.y, (unsigned)v.z, (unsigned)v.w};
      unsigned m = 0;
#pragma unroll
      for (int i = 0; i < 8; ++i) {
        const unsigned y = x[i];  // bytes b0..b3 in {0,1}
        m |= ((y & 1u) | ((y >> 7) & 2u) | ((y >> 14) & 4u) | ((y >> 21) & 8u)) << (4 * i);
      }
      if (wd == nw - 1 && (R & 31)) m &= (1u << (R & 31)) - 1u;  // bytes past R are stale
      if (bits) bits[wd] = m;
      cnt += __popc(m);
    }
    cnt = __reduce_add_sync(0xffffffffu, cnt);
    if (lane == 0) a.c_cnt[row] = cnt;
    __syncwarp();
  }
}

// Bitmap of every B row whose column range fits `bw` words: bbits[k * bw + w] bit b <=> column
// bmm[k].x + 32 w + b is in B row k.  (A B row referenced by a range row has range <= R_i, so
// rows wider than the range rows' R_max are never read.)  One warp per B row.
__global__ __launch_bounds__(256) void k_brow_bits(long long k, const int64_t* __restrict__ b_rpt,
                                                   const int32_t* __restrict__ b_col, const int2* __restrict__ bmm,
                                                   unsigned* __restrict__ bbits, int bw, int* __restrict__ wmax) {
  __shared__ unsigned s_w[8][64];
  const int lane = threadIdx.x & 31, wi = threadIdx.x >> 5;
  unsigned* sw = s_w[wi];
  int my_wmax = 0;
  for (long long row = (long long)blockIdx.x * 8 + wi; row < k; row += (long long)gridDim.x * 8) {
    const int2 mm = __ldg(bmm + row);
    if (mm.y < mm.x || (long long)mm.y - mm.x + 1 > 32LL * bw) continue;  // empty or too wide: unused
    const int nw = (mm.y - mm.x) / 32 + 1;
    my_wmax = max(my_wmax, nw);
    for (int w = lane; w < nw; w += 32) sw[w] = 0u;
    __syncwarp();
    const long long b0 = __ldg(b_rpt + row), b1 = __ldg(b_rpt + row + 1);
    for (long long j = b0 + lane; j < b1; j += 32) {
      const unsigned d = (unsigned)(__ldg(b_col + j) - mm.x);
      atomicOr(sw + (d >> 5), 1u << (d & 31));
    }
    __syncwarp();
    for (int w = lane; w < nw; w += 32) bbits[row * bw + w] = sw[w];
    __syncwarp();
  }
  if (lane == 0 && my_wmax > 0) atomicMax(wmax, my_wmax);
}

// Step (3) on range rows with R_max <= 1024, from the B-row bitmaps: the pattern of row i is the
// OR over its A non-zeros k of B row k's bitmap shifted by lo_k - lo_i (a bitmap union instead of
// one flag store per product — ~W_k/32 word operations per A non-zero instead of nnz(B_k)).
// Lane gl of a group of L = 32/H lanes owns output word gl; H A non-zeros are OR-ed at a time (H
// groups, L >= words of the row), the groups are OR-reduced at the end.  Writes nnz_i = popcount
// and the pattern bitmap (the numeric gather's input).
//
// When every B bitmap has <= 31 words (wmax, from k_brow_bits), the OR is done per A non-zero
// instead: LB = next_pow2(wmax + 1) lanes per non-zero (lane g produces output word q + g from B
// words g and g-1), 32/LB non-zeros per step, OR-ed into a per-warp shared row bitmap — fewer
// steps than owning all output words per lane group (cant: 5-word B rows in 9-word output rows:
// 4 non-zeros per step instead of 2).
__global__ __launch_bounds__(1024, 1) void k_sym_range_bits(SymArgs a, const unsigned* __restrict__ bbits, int bw,
                                                            const int2* __restrict__ bmm, const int* __restrict__ wmax) {
  __shared__ int4 s_meta[32][kMetaBatch];  // (B bitmap offset lo, hi, shift, words)
  __shared__ unsigned s_row[32][32];       // per-warp row bitmap (per-non-zero mode)
  __shared__ int s_next;
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  int4* meta = s_meta[w];
  unsigned* rowb = s_row[w];
  const unsigned mb = smem_u32(meta);
  const int wm = *wmax;
  const int lblog = wm + 1 <= 2 ? 1 : wm + 1 <= 4 ? 2 : wm + 1 <= 8 ? 3 : wm + 1 <= 16 ? 4 : 5;
  const bool per_nz = wm + 1 <= 16;  // else the output-word-owner loop below
  const RowQueue rq = row_queue(a.nrows, &s_next);
  for (long long r = rq.pop(lane); r >= 0; r = rq.pop(lane)) {
    const int row = a.rows[r];
    const int2 rr = __ldg(a.rlohi + row);
    const int lo = rr.x, R = rr.y - rr.x + 1;  // R <= 1024
    const int nw = (R + 31) >> 5;
    if (per_nz) {
      const int LB = 1 << lblog, g = lane & (LB - 1), hh = lane >> lblog, H = 32 >> lblog;
      if (lane < nw) rowb[lane] = 0u;
      const long long a0 = __ldg(a.a_rpt + row);
      const int na = (int)(__ldg(a.a_rpt + row + 1) - a0);
      const int32_t* __restrict__ ac = a.a_col + a0;
      for (int bb = 0; bb < na; bb += kMetaBatch) {
        const int j = bb + lane;
        int4 m = make_int4(0, 0, 0, 0);
        if (j < na) {
          const int kk = __ldg(ac + j);
          const int2 mm = __ldg(bmm + kk);
          if (mm.y >= mm.x) {
            const long long off = (long long)kk * bw;
            m = make_int4((int)(off & 0xffffffff), (int)(off >> 32), mm.x - lo, (mm.y - mm.x) / 32 + 1);
          }
        }
        meta[lane] = m;
        __syncwarp();
        const int cnt = min(kMetaBatch, na - bb);
#pragma unroll 1
        for (int e0 = 0; e0 < cnt; e0 += H) {
          const int e = e0 + hh;
          int4 me = make_int4(0, 0, 0, 0);
          if (e < cnt) asm volatile("ld.shared.v4.b32 {%0, %1, %2, %3}, [%4];"
                                    : "=r"(me.x), "=r"(me.y), "=r"(me.z), "=r"(me.w) : "r"(mb + 16u * e));
          const int q = me.z >> 5, sh = me.z & 31;
          const unsigned* bk = bbits + (((long long)me.y << 32) | (unsigned)me.x);
          const unsigned x = g < me.w ? __ldg(bk + g) : 0u;
          unsigned y = __shfl_up_sync(0xffffffffu, x, 1, LB);
          if (g == 0) y = 0u;
          const unsigned v = (x << sh) | (sh ? (y >> (32 - sh)) : 0u);
          if (v) atomicOr(rowb + q + g, v);
        }
        __syncwarp();
      }
      int cnt = 0;
      if (lane < nw) {
        const unsigned acc = rowb[lane];
        if (a.rbits) a.rbits[r * a.rwcap + lane] = acc;
        cnt = __popc(acc);
      }
      cnt = __reduce_add_sync(0xffffffffu, cnt);
      if (lane == 0) a.c_cnt[row] = cnt;
      __syncwarp();
      continue;
    }
    const int hlog = nw <= 8 ? 2 : (nw <= 16 ? 1 : 0);  // H = 1 << hlog A non-zeros at a time
    const int L = 32 >> hlog, gl = lane & (L - 1), h = lane >> (5 - hlog);
    const long long a0 = __ldg(a.a_rpt + row);
    const int na = (int)(__ldg(a.a_rpt + row + 1) - a0);
    const int32_t* __restrict__ ac = a.a_col + a0;
    unsigned acc = 0u;
    for (int bb = 0; bb < na; bb += kMetaBatch) {
      const int j = bb + lane;
      int4 m = make_int4(0, 0, 0, 0);  // words = 0: contributes nothing
      if (j < na) {
        const int kk = __ldg(ac + j);
        const int2 mm = __ldg(bmm + kk);
        if (mm.y >= mm.x) {
          const long long off = (long long)kk * bw;
          m = make_int4((int)(off & 0xffffffff), (int)(off >> 32), mm.x - lo, (mm.y - mm.x) / 32 + 1);
        }
      }
      meta[lane] = m;
      __syncwarp();
      const int cnt = min(kMetaBatch, na - bb);
#pragma unroll 1
      for (int e0 = 0; e0 < cnt; e0 += 1 << hlog) {
        const int e = e0 + h;
        int4 me = make_int4(0, 0, 0, 0);
        if (e < cnt) asm volatile("ld.shared.v4.b32 {%0, %1, %2, %3}, [%4];"
                                  : "=r"(me.x), "=r"(me.y), "=r"(me.z), "=r"(me.w) : "r"(mb + 16u * e));
        const int q = me.z >> 5, sh = me.z & 31;
        const int jj = gl - q;
        const unsigned* bk = bbits + (((long long)me.y << 32) | (unsigned)me.x);
        const unsigned x = (jj >= 0 && jj < me.w) ? __ldg(bk + jj) : 0u;
        unsigned y = __shfl_up_sync(0xffffffffu, x, 1, L);
        if (gl == 0) y = 0u;
        acc |= (x << sh) | (sh ? (y >> (32 - sh)) : 0u);
      }
      __syncwarp();
    }
    for (int o = L; o < 32; o <<= 1) acc |= __shfl_xor_sync(0xffffffffu, acc, o);
    int cnt = 0;
    if (lane < nw) {
      if (a.rbits) a.rbits[r * a.rwcap + lane] = acc;
      cnt = __popc(acc);
    }
    cnt = __reduce_add_sync(0xffffffffu, cnt);
    if (lane == 0) a.c_cnt[row] = cnt;
  }
}

// Step (7) on range rows: per warp RMetaW | acc[NC][rcap] (VT).
template <typename VT, int NC>
__global__ __launch_bounds__(1024, 1) void k_num_range(NumArgs a, int rcap) {
  extern __shared__ __align__(16) unsigned char rsm[];
  __shared__ int s_next;
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  constexpr int kMetaBytes = (int)sizeof(RMetaW<VT>);
  unsigned char* wb = rsm + (size_t)w * (kMetaBytes + (size_t)NC * rcap * sizeof(VT));
  RMetaW<VT>* meta = reinterpret_cast<RMetaW<VT>*>(wb);
  VT* acc = reinterpret_cast<VT*>(wb + kMetaBytes);
  const unsigned ab = smem_u32(acc);
  const unsigned cstride = (unsigned)(rcap * sizeof(VT));
  const VT* __restrict__ av = static_cast<const VT*>(a.a_val);
  const VT* __restrict__ bv = static_cast<const VT*>(a.b_val);
  VT* __restrict__ cval = static_cast<VT*>(a.c_val);
  const unsigned below = (1u << lane) - 1u;
  const RowQueue rq = row_queue(a.nrows, &s_next);
  for (long long r = rq.pop(lane); r >= 0; r = rq.pop(lane)) {
    const int row = a.rows[r];
    const int2 rr = __ldg(a.rlohi + row);
    const int lo = rr.x, R = rr.y - rr.x + 1;
    {
      int4* v4 = reinterpret_cast<int4*>(acc);
      const int nv = (int)(((long long)R * sizeof(VT) + 15) >> 4);
      for (int s = lane; s < nv; s += 32) v4[s] = make_int4(0, 0, 0, 0);
      if (NC == 2) {
        int4* v4b = reinterpret_cast<int4*>(acc + rcap);
        for (int s = lane; s < nv; s += 32) v4b[s] = make_int4(0, 0, 0, 0);
      }
    }
    __syncwarp();
    // slot of key in copy c: cb[c] + key * sizeof(VT)
    // (a bank-row padding of the slots, d + d/32, was measured slower: 0.344 -> 0.355 ms on cant)
    const unsigned cb0 = opaque(ab - (unsigned)lo * (unsigned)sizeof(VT));
    const unsigned cb1 = opaque(cb0 + cstride);
    range_products<true, VT>(a.a_rpt, a.a_col, av, a.b_rpt, a.b_col, bv, row, lane, meta,
                             [&](bool valid, int key, VT x, VT wv, int e, bool serial) {
      const unsigned s = ((NC == 2 && (e & 1)) ? cb1 : cb0) + (unsigned)key * (unsigned)sizeof(VT);
      if (NC == 2 && !serial) {
        // at most two B rows in this step, on different copies
        if (valid) RVec<VT>::st(s, fma(x, wv, RVec<VT>::ld(s)));
      } else {
        // apply the step's B rows one at a time (lane 0 holds the smallest e of the step)
        const int elo = __shfl_sync(0xffffffffu, e, 0);
        const int ehi = __reduce_max_sync(0xffffffffu, valid ? e : elo);
        for (int ee = elo; ee <= ehi; ++ee) {
          if (valid && e == ee) RVec<VT>::st(s, fma(x, wv, RVec<VT>::ld(s)));
          __syncwarp();
        }
      }
      __syncwarp();
    });
    // gather + sort: walk the symbolic bitmap of the row 32 columns at a time
    const long long c0 = a.c_rpt[row];
    const long long cn = a.c_rpt[row + 1] - c0;
    int32_t* __restrict__ cc = a.c_col + c0;
    VT* __restrict__ cv = cval + c0;
    const unsigned* __restrict__ bits = a.rbits + r * a.rwcap;
    int pos = 0;
    const int nw = (R + 31) >> 5;
    for (int wd = 0; wd < nw; ++wd) {
      const unsigned m = __ldg(bits + wd);
      if ((m >> lane) & 1u) {
        const int d = wd * 32 + lane;
        const int p = pos + __popc(m & below);
        VT v = acc[d];
        if (NC == 2) v += acc[rcap + d];
        if (p < cn) { cc[p] = lo + d; cv[p] = v; }
      }
      pos += __popc(m);
    }
    if (lane == 0 && pos != cn) atomicOr(a.err_flags, 2);
    __syncwarp();
  }
}

template <typename K>
int range_grid(K kernel, int threads, size_t smem, int num_sms, long long nrows, int warps) {
  int occ = 0;
  if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kernel, threads, smem) != cudaSuccess) {
    cudaGetLastError();
    occ = 1;
  }
  occ = occ < 1 ? 1 : occ;
  const long long need = (nrows + warps - 1) / warps;
  const long long cap = (long long)num_sms * occ;
  return (int)(need < cap ? need : cap);
}

template <typename K>
cudaError_t set_smem(K kernel, size_t smem, PerDevice& cache) {
  auto& configured = cache.here();
  if ((long long)smem <= configured.load()) return cudaSuccess;
  cudaError_t e = cudaFuncSetAttribute(kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e == cudaSuccess) configured.store((long long)smem);
  return e;
}

}  // namespace

// Warps per CTA for a per-warp table of `per_warp` bytes: <= 32, <= kRangeSmemBudget in total.
// fp64 numeric tables get twice the budget: measured Protein-like fp64 567 -> 738 GFLOPS, cant
// 653 -> 667 (96 -> 192 KB; fp32 unchanged across 96-192 KB).
int range_warps(long long per_warp, long long budget_default) {
  static const long long env = [] {
    const char* e = getenv("SPGEMM_RANGE_BUDGET");  // diagnostics: per-CTA table budget (bytes)
    return e ? atoll(e) : 0LL;
  }();
  const long long budget = env > 0 ? env : budget_default;
  long long w = per_warp > 0 ? budget / per_warp : 32;
  if (w > 32) w = 32;
  if (w < 1) w = 1;
  return (int)w;
}

int range_rcap(long long rmax) { return (int)((rmax + 31) & ~31LL); }
int range_wcap(long long rmax) { return (int)((rmax + 31) >> 5); }

cudaError_t launch_symbolic_range(cudaStream_t s, const SymArgs& a, int rmax, int num_sms) {
  if (a.nrows <= 0) return cudaSuccess;
  const int rcap = range_rcap(rmax);
  const long long per = (long long)sizeof(RMetaW<int>) + rcap;
  const int warps = range_warps(per);
  const size_t smem = (size_t)warps * per;
  static PerDevice configured;
  cudaError_t e = set_smem(k_sym_range, smem, configured);
  if (e != cudaSuccess) return e;
  const int grid = range_grid(k_sym_range, warps * 32, smem, num_sms, a.nrows, warps);
  k_sym_range<<<grid, warps * 32, smem, s>>>(a, rcap);
  return cudaGetLastError();
}

cudaError_t launch_brow_bits(cudaStream_t s, long long k, const int64_t* b_rpt, const int32_t* b_col,
                             const int2* bmm, unsigned* bbits, int bw, int* wmax, int num_sms) {
  if (k <= 0) return cudaSuccess;
  const long long want = (k + 7) / 8;
  const long long cap = (long long)num_sms * 8;
  k_brow_bits<<<(unsigned)(want < cap ? want : cap), 256, 0, s>>>(k, b_rpt, b_col, bmm, bbits, bw, wmax);
  return cudaGetLastError();
}

cudaError_t launch_symbolic_range_bits(cudaStream_t s, const SymArgs& a, const unsigned* bbits, int bw,
                                       const int2* bmm, const int* wmax, int num_sms) {
  if (a.nrows <= 0) return cudaSuccess;
  const int grid = range_grid(k_sym_range_bits, 1024, 0, num_sms, a.nrows, 32);
  k_sym_range_bits<<<grid, 1024, 0, s>>>(a, bbits, bw, bmm, wmax);
  return cudaGetLastError();
}

template <typename VT>
constexpr long long range_num_budget() { return sizeof(VT) == 8 ? 2 * kRangeSmemBudget : kRangeSmemBudget; }

template <typename VT, int NC>
static cudaError_t launch_num_range_t(cudaStream_t s, const NumArgs& a, int rcap, int num_sms) {
  const long long per = (long long)sizeof(RMetaW<VT>) + (long long)NC * rcap * sizeof(VT);
  const int warps = range_warps(per, range_num_budget<VT>());
  const size_t smem = (size_t)warps * per;
  static PerDevice configured;
  cudaError_t e = set_smem(k_num_range<VT, NC>, smem, configured);
  if (e != cudaSuccess) return e;
  const int grid = range_grid(k_num_range<VT, NC>, warps * 32, smem, num_sms, a.nrows, warps);
  k_num_range<VT, NC><<<grid, warps * 32, smem, s>>>(a, rcap);
  return cudaGetLastError();
}

// Two accumulator copies while they still allow >= 16 warps per CTA, else one.
template <typename VT>
static cudaError_t launch_num_range_v(cudaStream_t s, const NumArgs& a, int rmax, int num_sms) {
  const int rcap = range_rcap(rmax);
  const long long per2 = (long long)sizeof(RMetaW<VT>) + 2LL * rcap * sizeof(VT);
  if (range_warps(per2, range_num_budget<VT>()) >= 16) return launch_num_range_t<VT, 2>(s, a, rcap, num_sms);
  return launch_num_range_t<VT, 1>(s, a, rcap, num_sms);
}

cudaError_t launch_numeric_range(cudaStream_t s, bool fp64, const NumArgs& a, int rmax, int num_sms) {
  if (a.nrows <= 0) return cudaSuccess;
  return fp64 ? launch_num_range_v<double>(s, a, rmax, num_sms) : launch_num_range_v<float>(s, a, rmax, num_sms);
}

}  // namespace spg
