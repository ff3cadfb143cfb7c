// kernels_esc.cu — batched kernels for wide-span, weakly compressing rows (power-law graphs:
// R-MAT, webbase), B200 addition.
//
// One CTA takes a BATCH of R rows of one symbolic group (n_prod_i in (B/2, B], R*B = CAP =
// TPR*KP products) and flattens their products: thread t owns products t, t+TPR, ... of the
// batch, held in registers (all KP gathers issued before use).  Batching equalises the work per
// CTA and amortises the per-row fixed costs (barriers, scans) that dominate one-row-per-CTA
// kernels on rows of a few hundred products.
//
//   k_sym_batch  step (3): every product's column is inserted into its row's
//                hash table in shared memory — Alg. 5 (multiplicative hash of the key into t_size slots,
//                linear probing, atomicCAS from -1), t_size = 4*next_pow2(n_prod_i) (2* for the largest group) — and
//                nnz_i = the number of successful inserts.
//   k_num_esc    step (7): the paper accumulates into a hash table, gathers
//                the occupied slots and sorts them by a comparison rank ("each thread counts the
//                number of elements with smaller keys").  For rows whose products are ~all
//                distinct (n_prod_i <= ESC_PCT/100 * nnz_i) the table is nearly all fixed cost,
//                so this kernel orders the products themselves: each row's span [lo_i, hi_i] is
//                cut into next_pow2(n_prod_i) buckets of 2^s columns; a shared-memory counting
//                pass places every product in its bucket (histogram, exclusive scan, scatter; a
//                batch whose largest bucket is crowded splits its buckets by the next bits);
//                inside a bucket (about one product on average) each product takes the paper's
//                comparison rank (#smaller keys); the first product of each column is the entry
//                (a head) and sums the values of its column (working precision);
//                a scan of the distinct count per bucket plus the head's rank among the bucket's
//                distinct columns gives every entry its final position in C.  Output is compact
//                and sorted and written with coalesced stores.
#include <climits>

#include "spgemm_internal.cuh"

namespace spg {

namespace {

constexpr unsigned kFull = 0xffffffffu;

// 32-bit CTA exclusive scan; ws holds >= 32 ints.  Two barriers (the second protects ws from
// the next call).
template <int TPR>
__device__ __forceinline__ int esc_scan(int v, int* total, int* ws) {
  constexpr int NW = TPR / 32;
  const int l = threadIdx.x & 31, w = threadIdx.x >> 5;
  int x = v;
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    const int y = __shfl_up_sync(kFull, x, d);
    if (l >= d) x += y;
  }
  if (l == 31) ws[w] = x;
  __syncthreads();
  int s = l < NW ? ws[l] : 0;
#pragma unroll
  for (int d = 1; d < NW; d <<= 1) {
    const int y = __shfl_up_sync(kFull, s, d);
    if (l >= d) s += y;
  }
  const int base = __shfl_sync(kFull, s, (w + 31) & 31);
  *total = __shfl_sync(kFull, s, NW - 1);
  __syncthreads();
  return (w > 0 ? base : 0) + x - v;
}

// Per-batch row table (shared memory), filled by warp 0.
template <int R>
struct EscRows {
  long long a0[R];     // a_rpt[row]
  long long c0[R];     // c_rpt[row] (numeric)
  int lo[R];           // lowest column of the row's span
  int sh[R];           // bucket width 2^sh columns
  int ebase[R + 1];    // first A entry of the row in the batch's concatenated A entries
  int pbase[R + 1];    // first product / slot of the row
  int bbase[R + 1];    // first bucket (numeric) / first table slot / 4 (symbolic)
  int obase[R + 1];    // first output entry (numeric)
  int nr;              // rows in this batch
};

template <int R, bool NUM>
__device__ __forceinline__ void esc_rows(EscRows<R>* rt, const int32_t* __restrict__ rows, long long nrows,
                                         const int64_t* __restrict__ a_rpt, const int64_t* __restrict__ nprod,
                                         const int2* __restrict__ rlohi, const int64_t* __restrict__ c_rpt) {
  static_assert(R <= 32, "rows per batch");
  if (threadIdx.x >= 32) return;
  const int l = threadIdx.x;
  const long long gi = (long long)blockIdx.x * R + l;
  int na = 0, P = 0, nb = 0, nnz = 0, lo = 0, sh = 0;
  long long a0 = 0, c0 = 0;
  if (l < R && gi < nrows) {
    const int row = __ldg(rows + gi);
    a0 = __ldg(a_rpt + row);
    na = (int)(__ldg(a_rpt + row + 1) - a0);
    P = (int)__ldg(nprod + row);
    nb = P > 1 ? 1 << (32 - __clz(P - 1)) : 1;  // next_pow2(n_prod_i)
    if constexpr (NUM) {
      const int2 lh = __ldg(rlohi + row);
      lo = lh.x;
      const unsigned span = lh.y >= lh.x ? (unsigned)(lh.y - lh.x) : 0u;
      const int bits = span ? 32 - __clz(span) : 0;  // columns lo + [0, 2^bits)
      sh = max(0, bits - (31 - __clz(nb)));          // -> nb buckets of 2^sh columns
      c0 = c_rpt[row];
      nnz = (int)(c_rpt[row + 1] - c0);
    }
  }
  int e = na, p = P, b = nb, o = nnz;
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    const int ye = __shfl_up_sync(kFull, e, d), yp = __shfl_up_sync(kFull, p, d);
    const int yb = __shfl_up_sync(kFull, b, d), yo = __shfl_up_sync(kFull, o, d);
    if (l >= d) { e += ye; p += yp; b += yb; o += yo; }
  }
  if (l < R) {
    rt->a0[l] = a0; rt->c0[l] = c0; rt->lo[l] = lo; rt->sh[l] = sh;
    rt->ebase[l + 1] = e; rt->pbase[l + 1] = p; rt->bbase[l + 1] = b; rt->obase[l + 1] = o;
  }
  if (l == 0) {
    rt->ebase[0] = rt->pbase[0] = rt->bbase[0] = rt->obase[0] = 0;
    const long long left = nrows - (long long)blockIdx.x * R;
    rt->nr = (int)(left < R ? left : R);
  }
}

// Last r in [0, nr) with base[r] <= x (base ascending, base[0] = 0).
template <int R>
__device__ __forceinline__ int esc_find(const int* base, int nr, int x) {
  int lo = 0, hi = nr - 1;
#pragma unroll 1
  while (lo < hi) {
    const int mid = (lo + hi + 1) >> 1;
    if (base[mid] <= x) lo = mid; else hi = mid - 1;
  }
  return lo;
}

// Metadata of one chunk of the batch's A entries (shared memory).
template <typename VT, int ME, int CAP>
struct EscMeta {
  long long b0[ME];   // rpt_B[col_A]
  VT av[ME];          // val_A (numeric)
  int incl[ME];       // inclusive scan of the B-row lengths
  int bstart[CAP / 32 + 1];  // 32-product block -> first A entry holding one of its products
  uint8_t row[ME];    // batch row of the entry
};

// Gather of the batch's products into registers: key[u], val[u], rix[u] (batch row) for
// product p = t + u*TPR (key -1: none).  Metadata in chunks of ME A entries (MC per thread,
// contiguous); a chunk's products are located through the 32-product block-start table.
template <typename VT, bool NUM, int TPR, int KP, int MC, int R, int CAP>
__device__ __forceinline__ void esc_gather(const EscRows<R>* rt, EscMeta<VT, TPR * MC, CAP>* mt,
                                           const int32_t* __restrict__ a_col, const VT* __restrict__ a_val,
                                           const int64_t* __restrict__ b_rpt, const int32_t* __restrict__ b_col,
                                           const VT* __restrict__ b_val, int* ws, int (&key)[KP], VT (&val)[KP],
                                           int (&rix)[KP]) {
  constexpr int ME = TPR * MC;
  const int t = threadIdx.x;
  const int nr = rt->nr;
  const int E = rt->ebase[nr];
#pragma unroll
  for (int u = 0; u < KP; ++u) key[u] = -1;
  int pc0 = 0;
  for (int ec = 0; ec < E; ec += ME) {  // CTA-uniform
    int lens[MC];
    int mys = 0;
#pragma unroll
    for (int j = 0; j < MC; ++j) {
      const int e = t * MC + j, ge = ec + e;
      lens[j] = 0;
      if (ge < E) {
        const int r = esc_find<R>(rt->ebase, nr, ge);
        const long long ai = rt->a0[r] + (ge - rt->ebase[r]);
        const int kk = __ldg(a_col + ai);
        const long long b0 = __ldg(b_rpt + kk);
        lens[j] = (int)(__ldg(b_rpt + kk + 1) - b0);
        mt->b0[e] = b0;
        mt->row[e] = (uint8_t)r;
        if constexpr (NUM) mt->av[e] = __ldg(a_val + ai);
      }
      mys += lens[j];
    }
    int Pch;
    int run = esc_scan<TPR>(mys, &Pch, ws);
#pragma unroll
    for (int j = 0; j < MC; ++j) {
      const int e = t * MC + j;
      if (ec + e < E) {
        const int s = run, en = run + lens[j];
        mt->incl[e] = en;
        for (int k = (s + 31) >> 5; k < ((en + 31) >> 5); ++k) mt->bstart[k] = e;
        run = en;
      }
    }
    __syncthreads();
#pragma unroll
    for (int u = 0; u < KP; ++u) {
      const int lp = t + u * TPR - pc0;
      if (lp >= 0 && lp < Pch) {
        int e = mt->bstart[lp >> 5];
        while (mt->incl[e] <= lp) ++e;
        const long long q = mt->b0[e] + (lp - (e ? mt->incl[e - 1] : 0));
        key[u] = __ldg(b_col + q);
        if constexpr (NUM) val[u] = mt->av[e] * __ldg(b_val + q);
        rix[u] = mt->row[e];
      }
    }
    pc0 += Pch;
    __syncthreads();  // the next chunk rewrites the metadata
  }
}

// ---------------------------------------------------------------------------------------------
// Symbolic: batched paper hash (Alg. 5) per row.
template <int TPR, int KP, int MC, int R>
struct SymBatchSmem {
  static constexpr int CAP = TPR * KP;
  static constexpr int TF = CAP <= 8192 ? 4 : 2;  // table slots per product bound (load <= 1/TF)
  int tab[TF * CAP];  // per-row tables of TF*next_pow2(n_prod_i) slots
  EscMeta<int, TPR * MC, CAP> mt;
  EscRows<R> rt;
  int rcnt[R];
  int ws[32];
};

template <int TPR, int KP, int MC, int R>
__global__ __launch_bounds__(TPR) void k_sym_batch(SymArgs a) {
  using S = SymBatchSmem<TPR, KP, MC, R>;
  constexpr int CAP = S::CAP;
  extern __shared__ __align__(16) unsigned char smem_raw[];
  S* sm = reinterpret_cast<S*>(smem_raw);
  const int t = threadIdx.x, lane = t & 31;
  esc_rows<R, false>(&sm->rt, a.rows, a.nrows, a.a_rpt, a.nprod, nullptr, nullptr);
  {
    int4* tb = reinterpret_cast<int4*>(sm->tab);
    for (int i = t; i < S::TF * CAP / 4; i += TPR) tb[i] = make_int4(-1, -1, -1, -1);
    if (t < R) sm->rcnt[t] = 0;
  }
  __syncthreads();
  int key[KP], rix[KP];
  int dummy[KP];
  esc_gather<int, false, TPR, KP, MC, R, CAP>(&sm->rt, &sm->mt, a.a_col, nullptr, a.b_rpt, a.b_col, nullptr, sm->ws,
                                              key, dummy, rix);
  const unsigned tab = smem_u32(sm->tab);
#pragma unroll
  for (int u = 0; u < KP; ++u) {
    bool ins = false;
    const int r = key[u] >= 0 ? rix[u] : -1;
    if (r >= 0) {
      const int tb0 = S::TF * sm->rt.bbase[r];
      const unsigned mask = (unsigned)(S::TF * (sm->rt.bbase[r + 1] - sm->rt.bbase[r]) - 1);
      const SKeys K{tab + 4u * (unsigned)tb0};
      probe(K, mask, key[u], ins);
    }
    // nz++ per successful insert, aggregated per row across the warp
    const unsigned insm = __ballot_sync(kFull, ins);
    const int r0 = __shfl_sync(kFull, r, 0);
    if (__all_sync(kFull, r == r0 || r < 0)) {
      if (lane == 0 && insm) atomicAdd(&sm->rcnt[r0], __popc(insm));
    } else {
      const unsigned peers = __match_any_sync(kFull, r);
      if (r >= 0 && lane == __ffs(peers) - 1) {
        const int c = __popc(peers & insm);
        if (c) atomicAdd(&sm->rcnt[r], c);
      }
    }
  }
  __syncthreads();
  if (t < sm->rt.nr) a.c_cnt[__ldg(a.rows + (long long)blockIdx.x * R + t)] = sm->rcnt[t];
}

// ---------------------------------------------------------------------------------------------
// Numeric: expand, bucket, rank, compress in shared memory.
// Shared-memory index swizzles: arrays read both "blocked" (thread t owns KP consecutive slots)
// and "striped" (lane-consecutive) get one pad word per 32 (per 16 for 8-byte elements), so a
// blocked stride of KP in {8, 16} hits 32 distinct banks.
__device__ __forceinline__ int sw4(int j) { return j + (j >> 5); }
template <typename VT>
__device__ __forceinline__ int swv(int j) { return sizeof(VT) == 8 ? j + (j >> 4) : j + (j >> 5); }

#ifndef SPG_ESC_V3
#define SPG_ESC_V3 1
#endif
// Key / value slots of sk / sv are only ever read striped (lane-consecutive) or at scattered
// slots, never blocked, so they need no swizzle (the fine counters that alias sk keep sw4).
__device__ __forceinline__ int kix(int j) { return SPG_ESC_V3 ? j : sw4(j); }
template <typename VT>
__device__ __forceinline__ int vix(int j) { return SPG_ESC_V3 ? j : swv<VT>(j); }

#ifndef SPG_ESC_SKEW
#define SPG_ESC_SKEW 32
#endif
constexpr int kEscSkew = SPG_ESC_SKEW;  // a batch whose largest bucket holds more products is refined
// Shared memory of one batch, sized so that 48 warps fit on an SM (fp32: 1536 / TPR CTAs): the
// fine counters of the refinement live in sk (dead until the scatter), and the bucket table cnt
// carries, by phase: coarse counters -> starts -> fine base | bits << 24 (refinement) -> starts
// (low 16 bits) | duplicate count << 16 (rank) -> start | output base << 16 | has-duplicates << 31.
template <typename VT, int TPR, int KP, int MC, int R>
struct NumEscSmem {
  static constexpr int CAP = TPR * KP;
  static constexpr int NB = CAP;  // coarse (and fine) buckets per batch, at most
  int sk[CAP + CAP / 32 + 2];   // keys: bucket order, then the compacted output; fine counters
  VT sv[CAP + CAP / 16 + 1];    // values, same orders
  alignas(16) int cnt[NB + NB / 32 + 2];  // bucket table (above)
  uint16_t sb[CAP];             // bucket of each slot (bucket order); bit 15: the slot heads its key
  EscMeta<VT, TPR * MC, CAP> mt;
  EscRows<R> rt;
  int ws[32];
  int smax;
};

// Exclusive scan of n = N*TPR counters c[] (blocked, swizzled) in place; c[n] = total; the
// counts are returned in vals.
template <int TPR, int N>
__device__ __forceinline__ int esc_scan_counts(int* c, int* ws, int (&vals)[N]) {
  const int t = threadIdx.x;
  int s = 0;
#pragma unroll
  for (int i = 0; i < N; ++i) {
    vals[i] = c[sw4(t * N + i)];
    s += vals[i];
  }
  int tot;
  int run = esc_scan<TPR>(s, &tot, ws);
#pragma unroll
  for (int i = 0; i < N; ++i) {
    c[sw4(t * N + i)] = run;
    run += vals[i];
  }
  if (t == 0) c[sw4(N * TPR)] = tot;
  return tot;
}

#ifndef SPG_ESC64_OCC
#define SPG_ESC64_OCC 1280  // fp64 threads per SM (R-MAT s22 fp64: 1024 / MC 2 71.9 ms, 1280 / MC 1 67.5, 1536 75.5)
#endif
#ifndef SPG_ESC_OCC
#define SPG_ESC_OCC 1536
#endif
constexpr int kEscOcc = SPG_ESC_OCC;  // fp32 threads per SM the launch bounds ask for

template <typename VT, int TPR, int KP, int MC, int R>
__global__ __launch_bounds__(TPR, (sizeof(VT) == 8 ? SPG_ESC64_OCC : kEscOcc) / TPR) void k_num_esc(NumArgs a) {
  using S = NumEscSmem<VT, TPR, KP, MC, R>;
  constexpr int CAP = S::CAP;
  static_assert(CAP <= 4096, "bucket starts and output bases are packed into 16 and 15 bits");
  extern __shared__ __align__(16) unsigned char smem_raw[];
  S* sm = reinterpret_cast<S*>(smem_raw);
  const int t = threadIdx.x;
  esc_rows<R, true>(&sm->rt, a.rows, a.nrows, a.a_rpt, a.nprod, a.rlohi, a.c_rpt);
  {
    int4* c4 = reinterpret_cast<int4*>(sm->cnt);
    for (int i = t; i < (S::NB + S::NB / 32 + 2) / 4; i += TPR) c4[i] = make_int4(0, 0, 0, 0);
    for (int i = ((S::NB + S::NB / 32 + 2) / 4) * 4 + t; i < S::NB + S::NB / 32 + 2; i += TPR) sm->cnt[i] = 0;
  }
  if (t == 0) sm->smax = 0;
  __syncthreads();
  const int nr = sm->rt.nr;
  int key[KP], rix[KP];
  VT val[KP];
  esc_gather<VT, true, TPR, KP, MC, R, CAP>(&sm->rt, &sm->mt, a.a_col, static_cast<const VT*>(a.a_val), a.b_rpt,
                                            a.b_col, static_cast<const VT*>(a.b_val), sm->ws, key, val, rix);
  // coarse buckets: bkt = bbase_r + ((key - lo_r) >> sh_r), next_pow2(n_prod_i) per row; pos =
  // arrival order in the bucket
  unsigned bp[KP];
  bool bad = false;
#pragma unroll
  for (int u = 0; u < KP; ++u) {
    bp[u] = 0xffffffffu;
    if (key[u] >= 0) {
      const int r = rix[u];
      const unsigned d = (unsigned)(key[u] - sm->rt.lo[r]) >> sm->rt.sh[r];
      const int nbr = sm->rt.bbase[r + 1] - sm->rt.bbase[r];
      if (d < (unsigned)nbr) {
        const int bkt = sm->rt.bbase[r] + (int)d;
        const int pos = atomicAdd(&sm->cnt[sw4(bkt)], 1);
        bp[u] = ((unsigned)bkt << 16) | (unsigned)pos;
      } else {
        bad = true;  // a key outside the row's span: inputs changed since the symbolic phase
      }
    }
  }
  if (bad) atomicOr(a.err_flags, 2);
  __syncthreads();
  const int NBt = sm->rt.bbase[nr];
  const int Pt = sm->rt.pbase[nr];
  constexpr int KB = KP;  // counters per thread
  {
    int c[KB];
    esc_scan_counts<TPR, KB>(sm->cnt, sm->ws, c);
    int mx = 0;  // the largest bucket (from the counts the scan read; published by the barrier below)
#pragma unroll
    for (int i = 0; i < KB; ++i) mx = max(mx, c[i]);
    mx = __reduce_max_sync(kFull, mx);
    if ((t & 31) == 0 && mx > kEscSkew) atomicMax(&sm->smax, mx);
  }
  __syncthreads();
  if (sm->smax > kEscSkew) {
    // CTA-uniform: split each coarse bucket of n >= 2 products into 2^e fine buckets of the next
    // bits (down to single columns), e = ceil(log2 n) - 1, so that the fine buckets number at
    // most n_prod <= NB.  ep: 4 bits per coarse bucket of this thread (e, 15 = empty).
    unsigned long long ep = 0;
    int tot_f = 0;
#pragma unroll
    for (int i = 0; i < KB; ++i) {
      const int b = t * KB + i;
      const int n = sm->cnt[sw4(b + 1)] - sm->cnt[sw4(b)];
      int e = 15;
      if (b < NBt && n > 0) {
        e = 0;
        if (n > 1) {
          const int r = esc_find<R>(sm->rt.bbase, nr, b);
          e = min(31 - __clz(n - 1), sm->rt.sh[r]);
        }
        tot_f += 1 << e;
      }
      ep |= (unsigned long long)e << (4 * i);
    }
    int F;
    int run = esc_scan<TPR>(tot_f, &F, sm->ws);  // (every thread has read its counts before it)
    int* fcnt = sm->sk;  // fine counters (sk is dead until the scatter)
#pragma unroll
    for (int i = 0; i < KB; ++i) {
      const int e = (int)((ep >> (4 * i)) & 15u);
      sm->cnt[sw4(t * KB + i)] = run | ((e & 15) << 24);  // fine base of coarse bucket t*KB+i, bits
      if (e != 15) run += 1 << e;
    }
    for (int i = t; i < S::NB + S::NB / 32 + 2; i += TPR) fcnt[i] = 0;
    __syncthreads();
#pragma unroll
    for (int u = 0; u < KP; ++u)
      if (bp[u] != 0xffffffffu) {
        const int b = (int)(bp[u] >> 16), r = esc_find<R>(sm->rt.bbase, nr, b);  // (rix is dead here)
        const int fe = sm->cnt[sw4(b)];
        const int e = fe >> 24;
        const unsigned rel = (unsigned)(key[u] - sm->rt.lo[r]);
        const int fb = (fe & 0xffffff) + (int)((rel >> (sm->rt.sh[r] - e)) & ((1u << e) - 1u));
        const int pos = atomicAdd(&fcnt[sw4(fb)], 1);
        bp[u] = ((unsigned)fb << 16) | (unsigned)pos;
      }
    __syncthreads();
    int c2[KB];
    esc_scan_counts<TPR, KB>(fcnt, sm->ws, c2);
    __syncthreads();
    for (int i = t; i < S::NB + S::NB / 32 + 2; i += TPR) sm->cnt[i] = fcnt[i];
    __syncthreads();
  }
  int* const bst = sm->cnt;  // bucket starts (coarse, or fine after refinement)
  // scatter into bucket order (sb: the bucket of every slot)
#pragma unroll
  for (int u = 0; u < KP; ++u)
    if (bp[u] != 0xffffffffu) {
      const int b = (int)(bp[u] >> 16);
      const int slot = bst[sw4(b)] + (int)(bp[u] & 0xffffu);
      sm->sk[kix(slot)] = key[u];
      sm->sv[vix<VT>(slot)] = val[u];
      sm->sb[slot] = (uint16_t)b;
    }
  __syncthreads();
  // Inside the bucket, one slot per lane in bucket order (the lanes of a warp walk the same few
  // buckets together: uniform trip counts, broadcast reads): lt = #smaller keys (PAPER.md:173's
  // comparison rank), the slot heads its key when no equal key sits before it; a head sums the
  // values of all equal keys (accumulation in the working precision); a non-head
  // is counted as a duplicate of its bucket (high half of its bucket-table word).
  int lt[KP];
#pragma unroll
  for (int i = 0; i < KP; ++i) {
    const int j = i * TPR + t;
    lt[i] = -1;
    if (j < Pt) {
      const int b = sm->sb[j];
      const int j0 = bst[sw4(b)] & 0xffff, j1 = bst[sw4(b + 1)] & 0xffff;
      const int k = sm->sk[kix(j)];
      VT sum = VT(0);
      int l = 0, eqb = 0;
#if SPG_ESC_V3
      // branch-free pass (two slots per step): #smaller keys and #equal keys (itself included);
      // the values of equal keys are summed in a second pass only where a key repeats (rare for
      // weakly compressing rows)
      int ne = 0;
      int q = j0;
#pragma unroll 1
      for (; q + 1 < j1; q += 2) {
        const int k2 = sm->sk[q], k3 = sm->sk[q + 1];
        l += (k2 < k) + (k3 < k);
        ne += (k2 == k) + (k3 == k);
      }
      if (q < j1) {
        const int k2 = sm->sk[q];
        l += k2 < k;
        ne += k2 == k;
      }
      if (ne == 1) {
        sum = sm->sv[j];
      } else {
#pragma unroll 1
        for (int q2 = j0; q2 < j1; ++q2)
          if (sm->sk[q2] == k) {
            eqb += q2 < j;
            sum += sm->sv[q2];
          }
      }
#else
#pragma unroll 1
      for (int q = j0; q < j1; ++q) {
        const int k2 = sm->sk[sw4(q)];
        l += k2 < k;
        if (k2 == k) {  // (rare for weakly compressing rows, except q == j)
          eqb += q < j;
          sum += sm->sv[swv<VT>(q)];
        }
      }
#endif
      if (eqb == 0) {
        lt[i] = l;
        key[i] = k;
        val[i] = sum;
        sm->sb[j] = (uint16_t)(b | 0x8000);
      } else {
        atomicAdd(&bst[sw4(b)], 1 << 16);
      }
    }
  }
  __syncthreads();
  // distinct entries per bucket -> exclusive scan (blocked, KB buckets per thread) -> output base
  int H;
  {
    int s = 0;
    unsigned w0 = (unsigned)bst[sw4(t * KB)];
#pragma unroll
    for (int i = 0; i < KB; ++i) {
      const unsigned w1 = (unsigned)bst[sw4(t * KB + i + 1)];
      s += t * KB + i < NBt ? (int)(w1 & 0xffffu) - (int)(w0 & 0xffffu) - (int)(w0 >> 16) : 0;
      w0 = w1;
    }
    int run = esc_scan<TPR>(s, &H, sm->ws);  // (every thread has read its words before it)
    // (a thread rewrites only its own words, after reading them; the low halves stay)
    w0 = (unsigned)bst[sw4(t * KB)];
#pragma unroll
    for (int i = 0; i < KB; ++i) {
      const int b = t * KB + i;
      const unsigned w1 = (unsigned)bst[sw4(b + 1)], dup = w0 >> 16;
      bst[sw4(b)] = (int)((w0 & 0xffffu) | ((unsigned)run << 16) | (dup ? 0x80000000u : 0u));
      run += b < NBt ? (int)(w1 & 0xffffu) - (int)(w0 & 0xffffu) - (int)dup : 0;
      w0 = w1;
    }
  }
  const int Ot = sm->rt.obase[nr];
  const bool ok = H == Ot;  // CTA-uniform; false only when symbolic and numeric disagree
  if (!ok && t == 0) atomicOr(a.err_flags, 2);
  __syncthreads();
  // each head's position among the batch's distinct entries: its bucket's base + the number of
  // distinct smaller keys in the bucket (= lt when the bucket holds no equal keys)
#pragma unroll
  for (int i = 0; i < KP; ++i) {
    if (lt[i] >= 0) {
      const int j = i * TPR + t;
      const int b = sm->sb[j] & 0x7fff;
      const unsigned dbb = (unsigned)bst[sw4(b)];
      int dl = lt[i];
      if (dbb >> 31) {  // bucket with equal keys: count the smaller heads only
        const int j0 = (int)(dbb & 0xffffu), j1 = bst[sw4(b + 1)] & 0xffff;
        dl = 0;
#pragma unroll 1
        for (int q = j0; q < j1; ++q) dl += (sm->sk[kix(q)] < key[i]) & (sm->sb[q] >> 15);
      }
      lt[i] = (int)((dbb >> 16) & 0x7fffu) + dl;
    }
  }
  __syncthreads();
  if (ok) {
#pragma unroll
    for (int i = 0; i < KP; ++i)
      if (lt[i] >= 0) {
        sm->sk[kix(lt[i])] = key[i];
        sm->sv[vix<VT>(lt[i])] = val[i];
      }
  }
  __syncthreads();
  if (!ok) return;
  // coalesced copy of each row's compact, sorted entries to C (the row index advances with o)
  int32_t* __restrict__ cc = a.c_col;
  VT* __restrict__ cv = static_cast<VT*>(a.c_val);
  if constexpr (R == 1) {
    int32_t* __restrict__ c1 = cc + sm->rt.c0[0];
    VT* __restrict__ v1 = cv + sm->rt.c0[0];
    for (int o = t; o < Ot; o += TPR) {
      c1[o] = sm->sk[kix(o)];
      v1[o] = sm->sv[vix<VT>(o)];
    }
  } else {
    int r = t < Ot ? esc_find<R>(sm->rt.obase, nr, t) : 0;
    for (int o = t; o < Ot; o += TPR) {
      while (sm->rt.obase[r + 1] <= o) ++r;
      const long long dst = sm->rt.c0[r] + (o - sm->rt.obase[r]);
      cc[dst] = sm->sk[kix(o)];
      cv[dst] = sm->sv[vix<VT>(o)];
    }
  }
}

// ---------------------------------------------------------------------------------------------
// Per symbolic group (n_prod bound B): TPR threads, KP products per thread, R = KP*TPR/B rows per
// batch, MC A entries of metadata per thread per chunk.
struct EscCfg {
  int TPR, KP, MC;
};
// symbolic groups 2..9: bounds 128, 256, 512, 1024, 2048, 4096, 8192, 16384
constexpr EscCfg kEscSym[] = {{0, 0, 0}, {0, 0, 0}, {256, 8, 2},  {256, 8, 2},  {256, 8, 2},
                              {256, 8, 2}, {256, 8, 2}, {512, 8, 2}, {1024, 8, 2}, {1024, 16, 1}};
#ifndef SPG_ESC_SMALL_TPR
#define SPG_ESC_SMALL_TPR 128
#endif
constexpr int kEscSmallTpr = SPG_ESC_SMALL_TPR;
#ifndef SPG_ESC_KP
#define SPG_ESC_KP 8
#endif
#ifndef SPG_ESC_MC
#define SPG_ESC_MC 1
#endif
constexpr int kEscKp = SPG_ESC_KP;  // products per thread (fp32); CAP = TPR * KP >= the group bound
constexpr EscCfg kEscNum32[] = {{0, 0, 0},
                                {0, 0, 0},
                                {kEscSmallTpr, kEscKp, SPG_ESC_MC},
                                {kEscSmallTpr, kEscKp, SPG_ESC_MC},
                                {kEscSmallTpr, kEscKp, SPG_ESC_MC},
                                {kEscSmallTpr * 8 / kEscKp >= 128 ? kEscSmallTpr * 8 / kEscKp : 128, kEscKp, SPG_ESC_MC},
                                {256 * 8 / kEscKp, kEscKp, SPG_ESC_MC},
                                {512 * 8 / kEscKp, kEscKp, SPG_ESC_MC},
                                {1024, 8, 2},
                                {1024, 16, 1}};
#ifndef SPG_ESC64_TPR
#define SPG_ESC64_TPR 256
#endif
#ifndef SPG_ESC64_MC
#define SPG_ESC64_MC 1
#endif
constexpr int kEsc64Tpr = SPG_ESC64_TPR;  // fp64 groups 2-5 (group 6: max(256, this))
constexpr EscCfg kEscNum64[] = {{0, 0, 0},
                                {0, 0, 0},
                                {kEsc64Tpr, 8, SPG_ESC64_MC},
                                {kEsc64Tpr, 8, SPG_ESC64_MC},
                                {kEsc64Tpr, 8, SPG_ESC64_MC},
                                {kEsc64Tpr >= 128 ? kEsc64Tpr : 128, 8, SPG_ESC64_MC},
                                {256, 8, SPG_ESC64_MC},
                                {512, 8, SPG_ESC64_MC},
                                {1024, 8, 2},
                                {1024, 16, 1}};
template <typename VT>
constexpr EscCfg esc_num_cfg(int g) { return sizeof(VT) == 8 ? kEscNum64[g] : kEscNum32[g]; }

template <typename K>
cudaError_t esc_prepare(K kernel, int smem, PerDevice& cache) {
  auto& c = cache.here();
  if (smem > c.load()) {
    cudaError_t e = cudaFuncSetAttribute(kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    if (e != cudaSuccess) return e;
    e = cudaFuncSetAttribute(kernel, cudaFuncAttributePreferredSharedMemoryCarveout, 100);
    if (e != cudaSuccess) return e;
    c.store(smem);
  }
  return cudaSuccess;
}

template <int G>
cudaError_t launch_sym_batch_g(cudaStream_t s, const SymArgs& a) {
  constexpr EscCfg c = kEscSym[G];
  constexpr int R = c.TPR * c.KP / (int)kSymGroups[G].upper;
  static_assert(R >= 1 && R <= 32, "rows per batch");
  using S = SymBatchSmem<c.TPR, c.KP, c.MC, R>;
  constexpr int smem = (int)sizeof(S);
  static_assert(smem <= kSmemLimit - 1024, "symbolic batch smem");
  static PerDevice cache;
  cudaError_t e = esc_prepare(k_sym_batch<c.TPR, c.KP, c.MC, R>, smem, cache);
  if (e != cudaSuccess) return e;
  const long long grid = (a.nrows + R - 1) / R;
  k_sym_batch<c.TPR, c.KP, c.MC, R><<<(unsigned)grid, c.TPR, smem, s>>>(a);
  return cudaGetLastError();
}

template <typename VT, int G>
constexpr int num_esc_smem_g() {
  constexpr EscCfg c = esc_num_cfg<VT>(G);
  constexpr int R = c.TPR * c.KP / (int)kSymGroups[G].upper;
  return (int)sizeof(NumEscSmem<VT, c.TPR, c.KP, c.MC, R>);
}
constexpr int kEscSmemMax = kSmemLimit - 1024;

template <typename VT, int G>
cudaError_t launch_num_esc_g(cudaStream_t s, const NumArgs& a) {
  constexpr EscCfg c = esc_num_cfg<VT>(G);
  constexpr int R = c.TPR * c.KP / (int)kSymGroups[G].upper;
  static_assert(R >= 1 && R <= 32, "rows per batch");
  constexpr int smem = num_esc_smem_g<VT, G>();
  if constexpr (smem > kEscSmemMax) {
    return cudaErrorInvalidValue;  // the caller does not route these rows here (numeric_esc_supported)
  } else {
    static PerDevice cache;
    cudaError_t e = esc_prepare(k_num_esc<VT, c.TPR, c.KP, c.MC, R>, smem, cache);
    if (e != cudaSuccess) return e;
    const long long grid = (a.nrows + R - 1) / R;
    k_num_esc<VT, c.TPR, c.KP, c.MC, R><<<(unsigned)grid, c.TPR, smem, s>>>(a);
    return cudaGetLastError();
  }
}

}  // namespace

bool numeric_esc_supported(int sym_group, bool fp64) {
  switch (sym_group) {
#define SPG_G(I) \
  case I: return (fp64 ? num_esc_smem_g<double, I>() : num_esc_smem_g<float, I>()) <= kSmemLimit - 1024;
    SPG_G(2) SPG_G(3) SPG_G(4) SPG_G(5) SPG_G(6) SPG_G(7)
#undef SPG_G
    default: return false;
  }
}

cudaError_t launch_symbolic_batch(cudaStream_t s, int group, const SymArgs& a) {
  if (a.nrows <= 0) return cudaSuccess;
  switch (group) {
#define SPG_G(I) \
  case I: return launch_sym_batch_g<I>(s, a);
    SPG_G(2) SPG_G(3) SPG_G(4) SPG_G(5) SPG_G(6) SPG_G(7) SPG_G(8) SPG_G(9)
#undef SPG_G
    default: return cudaErrorInvalidValue;
  }
}

cudaError_t launch_numeric_esc(cudaStream_t s, int sym_group, bool fp64, const NumArgs& a) {
  if (a.nrows <= 0) return cudaSuccess;
  switch (sym_group) {
#define SPG_G(I) \
  case I: return fp64 ? launch_num_esc_g<double, I>(s, a) : launch_num_esc_g<float, I>(s, a);
    SPG_G(2) SPG_G(3) SPG_G(4) SPG_G(5) SPG_G(6) SPG_G(7)
#undef SPG_G
    default: return cudaErrorInvalidValue;
  }
}

}  // namespace spg
