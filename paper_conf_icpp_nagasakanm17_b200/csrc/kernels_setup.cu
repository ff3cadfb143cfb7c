// kernels_setup.cu — steps (1), (2), (4), (6) of PAPER.md:80 (Figure 1) on sm_100a:
//   k_nprod_group   Alg. 2 fused with the step-(2) group id + per-group
//                   histogram, CTA-aggregated before the global atomics.
//   k_group_scatter "the grouping is done by generating the array of gathered row indices
//                   corresponding to each group": warp-aggregated (MATCH.ANY)
//                   CTA-local ranks, one global atomic per group per CTA.
//   k_scan_*        step (4): inclusive prefix sum of nnz_i into rpt_C (3-kernel tile scan),
//                   the first kernel fused with the step-(6) grouping by nnz_i.
//   k_validate      optional O(nnz) input validation.
//   k_splits        n_prod-balanced row blocks for the multi-GPU driver.
#include <climits>

#include "spgemm_internal.cuh"

namespace spg {

namespace {

constexpr int kSetupThreads = 256;

__device__ __forceinline__ int group_of(long long key, const Bounds& bd) {
  int g = 0;
  while (g < bd.nbounds && key > bd.upper[g]) ++g;
  if (g < bd.min_group) g = bd.min_group;
  return g;
}

// Per-group row counts with warp-aggregated 32-bit shared atomics (MATCH.ANY on the group).
__device__ __forceinline__ void count_group(bool valid, int g, int* s_cnt) {
  const unsigned peers = __match_any_sync(0xffffffffu, valid ? g : -1);
  const int lane = threadIdx.x & 31;
  if (valid && lane == __ffs(peers) - 1) atomicAdd(&s_cnt[g], __popc(peers));
}

// Lanes per row of the setup kernels: power of two ~ mean row length / 4 in [1, 32], computed
// on the device from rpt[0] and rpt[rows] (CTA-uniform); rows longer than kLongPerLane * G entries
// go to the whole warp (power-law hub rows).
constexpr int kLongPerLane = 16;
__device__ __forceinline__ int setup_glog(const int64_t* __restrict__ rpt, long long rows) {
  const long long nnz = __ldg(rpt + rows) - __ldg(rpt);
  const long long avg = rows > 0 ? nnz / rows : 0;
  int g = 0;
  while (g < 5 && (4LL << g) * 2 <= avg) ++g;  // 2^g <= avg / 4
  return g;
}

// Column range of every B row: bmm[k] = {min col, max col} ({INT_MAX, -1} if empty), and the
// "some B row is not strictly increasing" flag.  G lanes per row (grid-stride over row blocks).
constexpr int kDeferLen = 512;  // rows longer than this: one warp each in k_*_long

// Warp-wide min/max and strictly-increasing check of B row [s0, s1), 8 loads (+8 predecessors)
// in flight per lane.
__device__ __forceinline__ void brow_warp(const int32_t* __restrict__ b_col, long long s0, long long s1, int lane,
                                          int& mn, int& mx, bool& bad) {
  int pmn = INT_MAX, pmx = -1;
  bool pbad = false;
  for (long long j = s0 + lane; j < s1; j += 8 * 32) {
    int c[8], pv[8];
#pragma unroll
    for (int u = 0; u < 8; ++u) {
      const long long q = j + 32 * u;
      c[u] = q < s1 ? __ldg(b_col + q) : 0;
      pv[u] = q < s1 && q > s0 ? __ldg(b_col + q - 1) : INT_MIN;
    }
#pragma unroll
    for (int u = 0; u < 8; ++u)
      if (j + 32 * u < s1) {
        pmn = min(pmn, c[u]); pmx = max(pmx, c[u]);
        pbad |= pv[u] != INT_MIN && c[u] <= pv[u];
      }
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    pmn = min(pmn, __shfl_xor_sync(0xffffffffu, pmn, o));
    pmx = max(pmx, __shfl_xor_sync(0xffffffffu, pmx, o));
  }
  mn = pmn; mx = pmx;
  bad = __any_sync(0xffffffffu, pbad);
}

__global__ __launch_bounds__(kSetupThreads) void k_brow_minmax(long long k, const int64_t* __restrict__ b_rpt,
                                                               const int32_t* __restrict__ b_col,
                                                               int2* __restrict__ bmm, int4* __restrict__ binfo,
                                                               int* __restrict__ unsorted,
                                                               int32_t* __restrict__ defer, int* __restrict__ ndefer) {
  const int glog = setup_glog(b_rpt, k);
  const int G = 1 << glog, lane = threadIdx.x & 31, gl = lane & (G - 1);
  const int rpc = kSetupThreads >> glog;
  bool bad = false;
  // Contiguous row slices (coalesced rpt loads).  Rows longer than kDeferLen go to a list and are
  // handled by k_*_long, one warp each: power-law generators cluster their hub rows, and a warp
  // walking several of them in series set the kernel time (webbase: 152 us; interleaving rows
  // over CTAs instead cost the short-row shapes their coalescing: cant 25 -> 31 us).
  const long long T = (long long)gridDim.x * rpc;
  constexpr bool ilv = false;
  for (long long base = 0; base < k; base += T) {
    const long long row = base + (ilv ? (long long)(threadIdx.x >> glog) * gridDim.x + blockIdx.x
                                      : (long long)blockIdx.x * rpc + (threadIdx.x >> glog));
    long long b0 = 0, b1 = 0;
    if (row < k) { b0 = __ldg(b_rpt + row); b1 = __ldg(b_rpt + row + 1); }
    const bool is_long = b1 - b0 > (long long)kLongPerLane * G;
    int mn = INT_MAX, mx = -1;
    if (!is_long) {
      // 4 entries per lane per step, all loads issued first; the predecessor of entry j (for the
      // strictly-increasing check) is the previous lane's entry (shuffle), or for lane 0 the last
      // lane's entry of the previous slot
      const unsigned gm = G >= 32 ? 0xffffffffu : (((1u << G) - 1u) << (lane & ~(G - 1)));
      int carry = INT_MIN;  // entry j-1 of lane 0's first slot (none before the row start)
      for (long long j = b0 + gl; j - gl < b1; j += 4 * G) {  // G-uniform trip count
        int c[4];
#pragma unroll
        for (int u = 0; u < 4; ++u) c[u] = j + u * G < b1 ? __ldg(b_col + j + u * G) : INT_MAX;
#pragma unroll
        for (int u = 0; u < 4; ++u) {
          const bool in = j + u * G < b1;
          int prev = __shfl_up_sync(gm, c[u], 1, G);
          const int last = __shfl_sync(gm, c[u], G - 1, G);
          if (gl == 0) prev = carry;
          carry = last;
          if (in) {
            mn = min(mn, c[u]); mx = max(mx, c[u]);
            bad |= prev != INT_MIN && c[u] <= prev;
          }
        }
      }
    }
    for (int o = G >> 1; o > 0; o >>= 1) {
      mn = min(mn, __shfl_xor_sync(0xffffffffu, mn, o));
      mx = max(mx, __shfl_xor_sync(0xffffffffu, mx, o));
    }
    unsigned longs = __ballot_sync(0xffffffffu, is_long && gl == 0);
    while (longs) {
      const int src = __ffs(longs) - 1;
      longs &= longs - 1;
      const long long s0 = __shfl_sync(0xffffffffu, b0, src), s1 = __shfl_sync(0xffffffffu, b1, src);
      if (defer && s1 - s0 > kDeferLen) {  // warp-uniform: deferred to k_brow_minmax_long
        if (lane == src) defer[atomicAdd(ndefer, 1)] = (int32_t)row;
        continue;
      }
      int pmn, pmx;
      bool pbad;
      brow_warp(b_col, s0, s1, lane, pmn, pmx, pbad);
      bad |= pbad && lane == src;
      if (lane == src) { mn = pmn; mx = pmx; }
    }
    if (row < k && gl == 0 && !(defer && is_long && b1 - b0 > kDeferLen)) {
      bmm[row] = make_int2(mn, mx);
      if (binfo) binfo[row] = make_int4(mn, mx, (int)(b1 - b0), 0);
    }
  }
  if (__any_sync(0xffffffffu, bad) && lane == 0) atomicOr(unsorted, 1);
}

// Deferred long B rows: one warp per row.
__global__ __launch_bounds__(kSetupThreads) void k_brow_minmax_long(const int64_t* __restrict__ b_rpt,
                                                                    const int32_t* __restrict__ b_col,
                                                                    int2* __restrict__ bmm, int4* __restrict__ binfo,
                                                                    int* __restrict__ unsorted,
                                                                    const int32_t* __restrict__ defer,
                                                                    const int* __restrict__ ndefer) {
  const int lane = threadIdx.x & 31;
  const int nw = gridDim.x * (kSetupThreads / 32);
  const int n = *ndefer;
  for (int i = blockIdx.x * (kSetupThreads / 32) + (threadIdx.x >> 5); i < n; i += nw) {
    const int row = defer[i];
    int mn, mx;
    bool bad;
    const long long r0 = __ldg(b_rpt + row), r1 = __ldg(b_rpt + row + 1);
    brow_warp(b_col, r0, r1, lane, mn, mx, bad);
    if (lane == 0) {
      bmm[row] = make_int2(mn, mx);
      if (binfo) binfo[row] = make_int4(mn, mx, (int)(r1 - r0), 0);
      if (bad) atomicOr(unsorted, 1);
    }
  }
}

// Warp-wide n_prod and column span of A row [s0, s1), 8 entries per lane in flight.
__device__ __forceinline__ void nprod_warp(const int32_t* __restrict__ a_col, const int64_t* __restrict__ b_rpt,
                                           const int2* __restrict__ bmm, const int4* __restrict__ binfo,
                                           long long s0, long long s1, int lane, long long& np, int& lo, int& hi) {
  long long part = 0;
  int plo = INT_MAX, phi = -1;
  for (long long j = s0 + lane; j < s1; j += 8 * 32) {
    int kk[8];
#pragma unroll
    for (int u = 0; u < 8; ++u) kk[u] = j + 32 * u < s1 ? __ldg(a_col + j + 32 * u) : -1;
#pragma unroll
    for (int u = 0; u < 8; ++u)
      if (kk[u] >= 0) {
        if (binfo) {  // one 16-byte gather: span and length of the B row
          const int4 r = __ldg(binfo + kk[u]);
          part += r.z; plo = min(plo, r.x); phi = max(phi, r.y);
        } else {
          part += __ldg(b_rpt + kk[u] + 1) - __ldg(b_rpt + kk[u]);
          if (bmm) { const int2 r = __ldg(bmm + kk[u]); plo = min(plo, r.x); phi = max(phi, r.y); }
        }
      }
  }
  np = (long long)warp_sum_u64((unsigned long long)part);
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    plo = min(plo, __shfl_xor_sync(0xffffffffu, plo, o));
    phi = max(phi, __shfl_xor_sync(0xffffffffu, phi, o));
  }
  lo = plo; hi = phi;
}

// Row outputs of step (1)/(2): n_prod, span, group id (Table I bounds, or the range-row group).
__device__ __forceinline__ int nprod_finish(long long row, long long np, int lo, int hi, int64_t* __restrict__ nprod,
                                            int2* __restrict__ rlohi, uint8_t* __restrict__ grp,
                                            int64_t* __restrict__ c_rpt, const Bounds& bd, bool b_ok, int& span_max) {
  int g = -1;
  nprod[row] = np;
  if (rlohi) rlohi[row] = make_int2(lo, hi);
  if (np == 0) {
    c_rpt[row + 1] = 0;  // reading R13: empty product row -> nnz 0, no kernel work
  } else {
    const long long R = (long long)hi - lo + 1;
    // range rows (kernels_range.cu): narrow exact column span, enough products for a warp
    if (b_ok && rlohi && np >= bd.range_min_np && np <= kRangeMaxNprod && R <= kRangeMaxSpan &&
        R <= kRangeSpanPerProd * np) {
      g = bd.range_group;
      span_max = max(span_max, (int)R);
    } else {
      g = group_of(np, bd);
    }
  }
  grp[row] = (uint8_t)(g < 0 ? 0xFF : g);
  return g;
}

// n_prod of every row (Alg. 2) with G lanes per row; also the column span [lo_i, hi_i] of row i
// of C (min/max over its A entries of the B-row ranges): exact, since every B column appears in
// C (kept structurally); the group id (Table I bounds, or the range-row group) and the per-group
// histogram (CTA-aggregated before the global atomics).
__global__ __launch_bounds__(kSetupThreads) void k_nprod_group(
    long long m, const int64_t* __restrict__ a_rpt, const int32_t* __restrict__ a_col,
    const int64_t* __restrict__ b_rpt, const int2* __restrict__ bmm, const int4* __restrict__ binfo,
    int64_t* __restrict__ nprod,
    int2* __restrict__ rlohi, uint8_t* __restrict__ grp, int64_t* __restrict__ c_rpt,
    DevAcc* __restrict__ acc, Bounds bd, int32_t* __restrict__ defer, int* __restrict__ ndefer) {
  __shared__ int s_cnt[kMaxGroups];
  __shared__ unsigned long long s_total, s_max;
  if (threadIdx.x < kMaxGroups) s_cnt[threadIdx.x] = 0;
  if (threadIdx.x == 0) { s_total = 0; s_max = 0; }
  __syncthreads();
  const int glog = setup_glog(a_rpt, m);
  const int G = 1 << glog, lane = threadIdx.x & 31, gl = lane & (G - 1);
  const int rpc = kSetupThreads >> glog;
  const bool b_ok = bd.range_group >= 0 && __ldg(b_rpt + bd.range_k) < (1LL << 31);
  unsigned long long tot = 0, mxnp = 0;
  int span_max = 0;
  const long long T = (long long)gridDim.x * rpc;  // contiguous slices, long rows deferred (see k_brow_minmax)
  constexpr bool ilv = false;
  for (long long base = 0; base < m; base += T) {
    const long long row = base + (ilv ? (long long)(threadIdx.x >> glog) * gridDim.x + blockIdx.x
                                      : (long long)blockIdx.x * rpc + (threadIdx.x >> glog));
    long long a0 = 0, a1 = 0;
    if (row < m) { a0 = __ldg(a_rpt + row); a1 = __ldg(a_rpt + row + 1); }
    const bool is_long = a1 - a0 > (long long)kLongPerLane * G;
    // Alg. 2: n_prod += rpt_B[col_A[j]+1] - rpt_B[col_A[j]], j in [rpt_A[i], rpt_A[i+1])
    long long np = 0;
    int lo = INT_MAX, hi = -1;
    if (!is_long) {  // col_A loads first, then the rpt_B / span gathers, 4 entries at a time
      for (long long j = a0 + gl; j < a1; j += 4 * G) {
        int kk[4];
#pragma unroll
        for (int u = 0; u < 4; ++u) kk[u] = j + u * G < a1 ? __ldg(a_col + j + u * G) : -1;
#pragma unroll
        for (int u = 0; u < 4; ++u)
          if (kk[u] >= 0) {
            if (binfo) {  // one 16-byte gather: span and length of the B row
              const int4 r = __ldg(binfo + kk[u]);
              np += r.z; lo = min(lo, r.x); hi = max(hi, r.y);
            } else {
              np += __ldg(b_rpt + kk[u] + 1) - __ldg(b_rpt + kk[u]);
              if (bmm) { const int2 r = __ldg(bmm + kk[u]); lo = min(lo, r.x); hi = max(hi, r.y); }
            }
          }
      }
    }
    for (int o = G >> 1; o > 0; o >>= 1) {
      np += __shfl_xor_sync(0xffffffffu, np, o);
      lo = min(lo, __shfl_xor_sync(0xffffffffu, lo, o));
      hi = max(hi, __shfl_xor_sync(0xffffffffu, hi, o));
    }
    unsigned longs = __ballot_sync(0xffffffffu, is_long && gl == 0);
    bool deferred = false;
    while (longs) {
      const int src = __ffs(longs) - 1;
      longs &= longs - 1;
      const long long s0 = __shfl_sync(0xffffffffu, a0, src), s1 = __shfl_sync(0xffffffffu, a1, src);
      if (defer && s1 - s0 > kDeferLen) {  // warp-uniform: deferred to k_nprod_long
        if (lane == src) {
          defer[atomicAdd(ndefer, 1)] = (int32_t)row;
          deferred = true;
        }
        continue;
      }
      long long part;
      int plo, phi;
      nprod_warp(a_col, b_rpt, bmm, binfo, s0, s1, lane, part, plo, phi);
      if (lane == src) { np = part; lo = plo; hi = phi; }
    }
    const bool lead = row < m && gl == 0 && !deferred;
    int g = -1;
    if (lead) {
      g = nprod_finish(row, np, lo, hi, nprod, rlohi, grp, c_rpt, bd, b_ok, span_max);
      tot += (unsigned long long)np;
      mxnp = max(mxnp, (unsigned long long)np);
    }
    count_group(g >= 0, g, s_cnt);
  }
  tot = warp_sum_u64(tot);
  mxnp = warp_max_u64(mxnp);
  span_max = __reduce_max_sync(0xffffffffu, span_max);
  if (lane == 0) {
    if (tot) atomicAdd(&s_total, tot);
    if (mxnp) atomicMax(&s_max, mxnp);
    if (span_max > 0) atomicMax(&acc->range_rmax, span_max);
  }
  __syncthreads();
  if (threadIdx.x < kMaxGroups && s_cnt[threadIdx.x]) atomicAdd(&acc->sym_rows[threadIdx.x], (unsigned long long)s_cnt[threadIdx.x]);
  if (threadIdx.x == 0) {
    if (s_total) atomicAdd(&acc->total_nprod, s_total);
    if (s_max) atomicMax(&acc->max_nprod, s_max);
  }
}

// Deferred long A rows of step (1)/(2): one warp per row, statistics straight to DevAcc.
__global__ __launch_bounds__(kSetupThreads) void k_nprod_long(const int64_t* __restrict__ a_rpt,
                                                              const int32_t* __restrict__ a_col,
                                                              const int64_t* __restrict__ b_rpt,
                                                              const int2* __restrict__ bmm,
                                                              const int4* __restrict__ binfo, int64_t* __restrict__ nprod,
                                                              int2* __restrict__ rlohi, uint8_t* __restrict__ grp,
                                                              int64_t* __restrict__ c_rpt, DevAcc* __restrict__ acc,
                                                              Bounds bd, const int32_t* __restrict__ defer,
                                                              const int* __restrict__ ndefer) {
  const int lane = threadIdx.x & 31;
  const int nw = gridDim.x * (kSetupThreads / 32);
  const int n = *ndefer;
  const bool b_ok = bd.range_group >= 0 && __ldg(b_rpt + bd.range_k) < (1LL << 31);
  for (int i = blockIdx.x * (kSetupThreads / 32) + (threadIdx.x >> 5); i < n; i += nw) {
    const int row = defer[i];
    long long np;
    int lo, hi;
    nprod_warp(a_col, b_rpt, bmm, binfo, __ldg(a_rpt + row), __ldg(a_rpt + row + 1), lane, np, lo, hi);
    if (lane == 0) {
      int span_max = 0;
      const int g = nprod_finish(row, np, lo, hi, nprod, rlohi, grp, c_rpt, bd, b_ok, span_max);
      if (g >= 0) atomicAdd(&acc->sym_rows[g], 1ull);
      if (np) {
        atomicAdd(&acc->total_nprod, (unsigned long long)np);
        atomicMax(&acc->max_nprod, (unsigned long long)np);
      }
      if (span_max > 0) atomicMax(&acc->range_rmax, span_max);
    }
  }
}

constexpr int kScatterItems = 4;

__global__ __launch_bounds__(kSetupThreads) void k_group_scatter(long long m, const uint8_t* __restrict__ grp,
                                                                 Offsets off, int* __restrict__ cursor,
                                                                 int32_t* __restrict__ perm) {
  __shared__ int s_cnt[kMaxGroups], s_base[kMaxGroups];
  if (threadIdx.x < kMaxGroups) s_cnt[threadIdx.x] = 0;
  __syncthreads();
  const int lane = threadIdx.x & 31;
  int g[kScatterItems], local[kScatterItems];
  long long rowv[kScatterItems];
#pragma unroll
  for (int it = 0; it < kScatterItems; ++it) {
    const long long row = ((long long)blockIdx.x * kScatterItems + it) * kSetupThreads + threadIdx.x;
    rowv[it] = row;
    g[it] = row < m ? grp[row] : 0xFF;
    const unsigned peers = __match_any_sync(0xffffffffu, g[it]);
    const int leader = __ffs(peers) - 1;
    const int rank = __popc(peers & ((1u << lane) - 1u));
    int base = 0;
    if (lane == leader && g[it] != 0xFF) base = atomicAdd(&s_cnt[g[it]], __popc(peers));
    base = __shfl_sync(0xffffffffu, base, leader);
    local[it] = base + rank;
  }
  __syncthreads();
  if (threadIdx.x < off.ngroups && s_cnt[threadIdx.x])
    s_base[threadIdx.x] = atomicAdd(&cursor[threadIdx.x], s_cnt[threadIdx.x]);
  __syncthreads();
#pragma unroll
  for (int it = 0; it < kScatterItems; ++it)
    if (g[it] != 0xFF) perm[off.off[g[it]] + s_base[g[it]] + local[it]] = (int32_t)rowv[it];
}

// ------------------------------------------------------------------ scan (+ step-6 grouping)
constexpr int kScanItems = 8;
constexpr int kScanTile = kSetupThreads * kScanItems;

__device__ __forceinline__ long long block_sum_ll(long long v, long long* ws) {
  return Grp<kSetupThreads>::sum(v, ws);
}

// Tile reduction of x[0..m) (x = rpt_C + 1 holding nnz_i), fused with grouping by nnz_i
// (group ids, per-group row counts and the maximum nnz_i: what the host needs at sync 2).
__global__ __launch_bounds__(kSetupThreads) void k_scan_reduce(long long m, const int64_t* __restrict__ x,
                                                               long long* __restrict__ tile_sums,
                                                               const uint8_t* __restrict__ grp1,
                                                               uint8_t* __restrict__ grp2, DevAcc* __restrict__ acc,
                                                               Bounds bd, EscSel esc) {
  __shared__ long long ws[33];
  __shared__ int s_cnt[kMaxGroups];
  __shared__ unsigned long long s_max;
  const bool grouping = grp2 != nullptr;
  if (grouping) {
    if (threadIdx.x < kMaxGroups) s_cnt[threadIdx.x] = 0;
    if (threadIdx.x == 0) s_max = 0;
    __syncthreads();
  }
  const long long base = (long long)blockIdx.x * kScanTile;
  long long s = 0;
  unsigned long long mx = 0;
#pragma unroll
  for (int e = 0; e < kScanItems; ++e) {
    const long long i = base + e * kSetupThreads + threadIdx.x;
    const long long v = i < m ? x[i] : 0;
    s += v;
    if (grouping) {  // block-uniform branch
      int g = -1;
      if (i < m) {
        if (v > 0) {
          const int g1 = grp1[i];
          if (bd.range_group >= 0 && g1 == kSymRange) g = bd.range_group;
          else if (esc.nprod && g1 >= kEscSymLo && g1 <= kEscSymHi && ((esc.groups >> g1) & 1u) &&
                   100 * esc.nprod[i] <= (long long)esc.pct * v)
            g = kNumEscBase + g1 - kEscSymLo;
          else g = group_of(v, bd);
        }
        grp2[i] = (uint8_t)(g < 0 ? 0xFF : g);
      }
      count_group(g >= 0, g, s_cnt);
      mx = (unsigned long long)v > mx ? (unsigned long long)v : mx;
    }
  }
  const long long tot = block_sum_ll(s, ws);
  if (threadIdx.x == 0) tile_sums[blockIdx.x] = tot;
  if (grouping) {
    mx = warp_max_u64(mx);
    if ((threadIdx.x & 31) == 0 && mx) atomicMax(&s_max, mx);
    __syncthreads();
    if (threadIdx.x < kMaxGroups && s_cnt[threadIdx.x])
      atomicAdd(&acc->num_rows[threadIdx.x], (unsigned long long)s_cnt[threadIdx.x]);
    if (threadIdx.x == 0 && s_max) atomicMax(&acc->max_nnz, s_max);
  }
}

// Per-group sums for spgemm_get_stats (n_prod, nnz(A), nnz(C) of each group's rows): run on
// demand, off the SpGEMM critical path.
__global__ __launch_bounds__(kSetupThreads) void k_group_stats(long long m, const uint8_t* __restrict__ grp1,
                                                               const uint8_t* __restrict__ grp2,
                                                               const int64_t* __restrict__ nprod,
                                                               const int64_t* __restrict__ a_rpt,
                                                               const int64_t* __restrict__ c_rpt, DevAcc* acc) {
  __shared__ unsigned long long s[5][kMaxGroups];
  for (int i = threadIdx.x; i < 5 * kMaxGroups; i += blockDim.x) (&s[0][0])[i] = 0;
  __syncthreads();
  const long long i = (long long)blockIdx.x * kSetupThreads + threadIdx.x;
  int g1 = -1, g2 = -1;
  unsigned long long np = 0, na = 0, nc = 0;
  if (i < m) {
    g1 = grp1[i] == 0xFF ? -1 : grp1[i];
    g2 = grp2[i] == 0xFF ? -1 : grp2[i];
    np = (unsigned long long)nprod[i];
    na = (unsigned long long)(a_rpt[i + 1] - a_rpt[i]);
    nc = (unsigned long long)(c_rpt[i + 1] - c_rpt[i]);
  }
  {
    const unsigned long long v[2] = {np, na};
    unsigned long long* const d[2] = {s[0], s[1]};
    warp_group_add<2>(g1 >= 0, g1, v, d);
  }
  {
    const unsigned long long v[3] = {np, na, nc};
    unsigned long long* const d[3] = {s[2], s[3], s[4]};
    warp_group_add<3>(g2 >= 0, g2, v, d);
  }
  __syncthreads();
  if (threadIdx.x < kMaxGroups) {
    const int g = threadIdx.x;
    if (s[0][g]) atomicAdd(&acc->sym_nprod[g], s[0][g]);
    if (s[1][g]) atomicAdd(&acc->sym_nnza[g], s[1][g]);
    if (s[2][g]) atomicAdd(&acc->num_nprod[g], s[2][g]);
    if (s[3][g]) atomicAdd(&acc->num_nnza[g], s[3][g]);
    if (s[4][g]) atomicAdd(&acc->num_nnzc[g], s[4][g]);
  }
}

// Exclusive scan of the tile sums, one CTA of 1024 threads, carried across chunks.
__global__ __launch_bounds__(1024) void k_scan_tiles(long long ntiles, long long* __restrict__ t) {
  __shared__ long long ws[33];
  long long carry = 0;
  for (long long c = 0; c < ntiles; c += 1024) {
    const long long i = c + threadIdx.x;
    const long long v = i < ntiles ? t[i] : 0;
    long long tot;
    const long long ex = Grp<1024>::excl_scan(v, &tot, ws);
    if (i < ntiles) t[i] = carry + ex;
    carry += tot;
    __syncthreads();
  }
}

// In-place inclusive scan of each tile plus its offset.  Blocked arrangement: thread owns
// kScanItems consecutive elements.
__global__ __launch_bounds__(kSetupThreads) void k_scan_down(long long m, int64_t* __restrict__ x,
                                                             const long long* __restrict__ tile_off,
                                                             long long* __restrict__ total_out) {
  __shared__ long long ws[33];
  const long long base = (long long)blockIdx.x * kScanTile + (long long)threadIdx.x * kScanItems;
  long long v[kScanItems];
  long long s = 0;
#pragma unroll
  for (int e = 0; e < kScanItems; ++e) {
    const long long i = base + e;
    v[e] = i < m ? x[i] : 0;
    s += v[e];
  }
  long long tot;
  long long run = Grp<kSetupThreads>::excl_scan(s, &tot, ws) + tile_off[blockIdx.x];
#pragma unroll
  for (int e = 0; e < kScanItems; ++e) {
    const long long i = base + e;
    run += v[e];
    if (i < m) {
      x[i] = run;
      if (i == m - 1 && total_out) *total_out = run;
    }
  }
}

// One-CTA inclusive scan of x[0..m) for small m (the small-matrix path): one launch instead of
// three; chunks of 4096 staged through shared memory with coalesced loads and stores, a running
// carry across chunks.
constexpr int kSmallScanChunk = 4096;
// host_acc != nullptr: afterwards the CTA copies the whole DevAcc `acc` (the total included) to
// host_acc, pinned host memory the kernel writes through PCIe (no separate D2H copy node).
__global__ __launch_bounds__(1024) void k_scan_small(long long m, int64_t* __restrict__ x,
                                                     long long* __restrict__ total_out, const DevAcc* acc,
                                                     DevAcc* host_acc) {
  __shared__ long long tile[kSmallScanChunk];
  __shared__ long long ws[33];
  constexpr int PER = kSmallScanChunk / 1024;
  long long carry = 0;
  for (long long c = 0; c < m; c += kSmallScanChunk) {
#pragma unroll
    for (int e = 0; e < PER; ++e) {
      const long long i = c + e * 1024 + threadIdx.x;
      tile[e * 1024 + threadIdx.x] = i < m ? x[i] : 0;
    }
    __syncthreads();
    long long v[PER], s = 0;
#pragma unroll
    for (int e = 0; e < PER; ++e) {
      v[e] = tile[threadIdx.x * PER + e];
      s += v[e];
    }
    long long tot;
    long long run = carry + Grp<1024>::excl_scan(s, &tot, ws);
#pragma unroll
    for (int e = 0; e < PER; ++e) {
      run += v[e];
      tile[threadIdx.x * PER + e] = run;
    }
    __syncthreads();
#pragma unroll
    for (int e = 0; e < PER; ++e) {
      const long long i = c + e * 1024 + threadIdx.x;
      if (i < m) x[i] = tile[e * 1024 + threadIdx.x];
    }
    carry += tot;
    __syncthreads();
  }
  if (threadIdx.x == 0 && total_out) *total_out = carry;
  if (host_acc) {
    __syncthreads();  // the total above, the counters of the previous kernels
    static_assert(sizeof(DevAcc) % 4 == 0, "DevAcc words");
    const unsigned* src = reinterpret_cast<const unsigned*>(acc);
    unsigned* dst = reinterpret_cast<unsigned*>(host_acc);
    for (int i = threadIdx.x; i < (int)(sizeof(DevAcc) / 4); i += 1024) dst[i] = src[i];
  }
}

// ------------------------------------------------------------------ validation
__global__ void k_validate(long long m, long long k, long long n, const int64_t* __restrict__ a_rpt,
                           const int32_t* __restrict__ a_col, const int64_t* __restrict__ b_rpt,
                           const int32_t* __restrict__ b_col, int* __restrict__ err) {
  const long long stride = (long long)gridDim.x * blockDim.x;
  const long long tid = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  bool bad = false;
  for (long long i = tid; i < m; i += stride) bad |= a_rpt[i + 1] < a_rpt[i];
  for (long long i = tid; i < k; i += stride) bad |= b_rpt[i + 1] < b_rpt[i];
  const long long a0 = a_rpt[0], a1 = a_rpt[m], b0 = b_rpt[0], b1 = b_rpt[k];
  if (a0 < 0 || b0 < 0) bad = true;
  for (long long j = a0 + tid; j < a1; j += stride) { const int c = a_col[j]; bad |= (c < 0 || c >= k); }
  for (long long j = b0 + tid; j < b1; j += stride) { const int c = b_col[j]; bad |= (c < 0 || c >= n); }
  if (bad) atomicOr(err, 1);
}

// n_prod only (no grouping) for the partition.
__global__ __launch_bounds__(kSetupThreads) void k_nprod_only(long long m, const int64_t* __restrict__ a_rpt,
                                                              const int32_t* __restrict__ a_col,
                                                              const int64_t* __restrict__ b_rpt,
                                                              int64_t* __restrict__ out) {
  const long long row = (long long)blockIdx.x * (kSetupThreads / 32) + threadIdx.x / 32;
  const int l = threadIdx.x & 31;
  long long np = 0;
  if (row < m)
    for (long long j = a_rpt[row] + l; j < a_rpt[row + 1]; j += 32) {
      const int kk = a_col[j];
      np += b_rpt[kk + 1] - b_rpt[kk];
    }
#pragma unroll
  for (int off = 16; off > 0; off >>= 1) np += __shfl_xor_sync(0xffffffffu, np, off);
  if (row < m && l == 0) out[row] = np;
}

// splits[p] = min{ r in [0,m] : sum_{i<r} n_prod_i >= p*total/P }, splits[P] = m.
__global__ void k_splits(long long m, const int64_t* __restrict__ excl, int nparts, int64_t* __restrict__ splits) {
  const int p = blockIdx.x * blockDim.x + threadIdx.x;
  if (p > nparts) return;
  if (p == nparts) { splits[p] = m; return; }
  const long long total = excl[m];
  const long long target = (long long)((__int128)total * p / nparts);
  long long lo = 0, hi = m;
  while (lo < hi) {
    const long long mid = (lo + hi) / 2;
    if (excl[mid] >= target) hi = mid; else lo = mid + 1;
  }
  splits[p] = lo;
}

}  // namespace

cudaError_t launch_nprod_group(cudaStream_t s, long long m, long long k, const int64_t* a_rpt,
                               const int32_t* a_col, const int64_t* b_rpt, const int32_t* b_col, int2* bmm, int4* binfo,
                               int64_t* nprod, int2* rlohi, uint8_t* grp, int64_t* c_rpt, DevAcc* acc, Bounds b,
                               int32_t* defer_a, int32_t* defer_b, int* nlaunch) {
  if (m == 0) return cudaSuccess;
  // grid-stride kernels: enough CTAs for any lanes-per-row choice (rows / 8 per CTA-pass at G = 32)
  auto grid_of = [](long long rows) {
    const long long want = (rows + (kSetupThreads / 32) - 1) / (kSetupThreads / 32);
    return (unsigned)(want < 148LL * 16 ? (want > 0 ? want : 1) : 148LL * 16);
  };
  // deferred long rows (> kDeferLen entries): one warp each, 148 x 4 CTAs of 8 warps
  const unsigned long_grid = 148 * 4;
  if (bmm && k > 0) {
    k_brow_minmax<<<grid_of(k), kSetupThreads, 0, s>>>(k, b_rpt, b_col, bmm, binfo, &acc->b_unsorted, defer_b,
                                                       &acc->defer_count[0]);
    k_brow_minmax_long<<<long_grid, kSetupThreads, 0, s>>>(b_rpt, b_col, bmm, binfo, &acc->b_unsorted, defer_b,
                                                           &acc->defer_count[0]);
    if (nlaunch) *nlaunch += 2;
  }
  if (!(bmm && k > 0)) binfo = nullptr;  // only k_brow_minmax fills it
  k_nprod_group<<<grid_of(m), kSetupThreads, 0, s>>>(m, a_rpt, a_col, b_rpt, bmm, binfo, nprod, rlohi, grp, c_rpt, acc, b,
                                                     defer_a, &acc->defer_count[1]);
  k_nprod_long<<<long_grid, kSetupThreads, 0, s>>>(a_rpt, a_col, b_rpt, bmm, binfo, nprod, rlohi, grp, c_rpt, acc, b, defer_a,
                                                   &acc->defer_count[1]);
  if (nlaunch) *nlaunch += 2;
  return cudaGetLastError();
}

cudaError_t launch_group_stats(cudaStream_t s, long long m, const uint8_t* grp1, const uint8_t* grp2,
                               const int64_t* nprod, const int64_t* a_rpt, const int64_t* c_rpt, DevAcc* acc) {
  if (m == 0) return cudaSuccess;
  k_group_stats<<<(unsigned)((m + kSetupThreads - 1) / kSetupThreads), kSetupThreads, 0, s>>>(m, grp1, grp2, nprod,
                                                                                             a_rpt, c_rpt, acc);
  return cudaGetLastError();
}

cudaError_t launch_group_scatter(cudaStream_t s, long long m, const uint8_t* grp, Offsets off, int* cursor,
                                 int32_t* perm) {
  if (m == 0) return cudaSuccess;
  const long long per = (long long)kSetupThreads * kScatterItems;
  k_group_scatter<<<(unsigned)((m + per - 1) / per), kSetupThreads, 0, s>>>(m, grp, off, cursor, perm);
  return cudaGetLastError();
}

size_t scan_workspace_bytes(long long m) {
  return (size_t)((m + kScanTile - 1) / kScanTile + 1) * sizeof(long long);
}

static cudaError_t scan_inclusive(cudaStream_t s, long long m, int64_t* x, const uint8_t* grp1, uint8_t* grp2,
                                  DevAcc* acc, Bounds b, EscSel esc, long long* tile_ws, long long* total_out,
                                  int* nlaunch) {
  if (m == 0) return cudaSuccess;
  const long long ntiles = (m + kScanTile - 1) / kScanTile;
  k_scan_reduce<<<(unsigned)ntiles, kSetupThreads, 0, s>>>(m, x, tile_ws, grp1, grp2, acc, b, esc);
  k_scan_tiles<<<1, 1024, 0, s>>>(ntiles, tile_ws);
  k_scan_down<<<(unsigned)ntiles, kSetupThreads, 0, s>>>(m, x, tile_ws, total_out);
  if (nlaunch) *nlaunch += 3;
  return cudaGetLastError();
}

cudaError_t launch_scan_and_group(cudaStream_t s, long long m, int64_t* c_rpt, const uint8_t* grp1,
                                  uint8_t* grp2, DevAcc* acc, Bounds b, EscSel esc, long long* tile_ws,
                                  int* nlaunch) {
  return scan_inclusive(s, m, c_rpt + 1, grp1, grp2, acc, b, esc, tile_ws, &acc->nnzc, nlaunch);
}

cudaError_t launch_scan_small(cudaStream_t s, long long m, int64_t* c_rpt, DevAcc* acc, DevAcc* host_acc) {
  if (m <= 0) return cudaSuccess;
  k_scan_small<<<1, 1024, 0, s>>>(m, c_rpt + 1, &acc->nnzc, acc, host_acc);
  return cudaGetLastError();
}

cudaError_t launch_validate(cudaStream_t s, long long m, long long k, long long n, const int64_t* a_rpt,
                            const int32_t* a_col, const int64_t* b_rpt, const int32_t* b_col, int* err) {
  k_validate<<<1184, 256, 0, s>>>(m, k, n, a_rpt, a_col, b_rpt, b_col, err);
  return cudaGetLastError();
}

cudaError_t launch_partition(cudaStream_t s, long long m, const int64_t* a_rpt, const int32_t* a_col,
                             const int64_t* b_rpt, int64_t* nprod_scan, long long* tile_ws, int nparts,
                             int64_t* splits_dev, int* nlaunch) {
  cudaError_t e = cudaMemsetAsync(nprod_scan, 0, sizeof(int64_t), s);
  if (e != cudaSuccess) return e;
  if (m > 0) {
    const long long rpb = kSetupThreads / 32;
    k_nprod_only<<<(unsigned)((m + rpb - 1) / rpb), kSetupThreads, 0, s>>>(m, a_rpt, a_col, b_rpt, nprod_scan + 1);
    Bounds none{};
    none.range_group = -1;
    e = scan_inclusive(s, m, nprod_scan + 1, nullptr, nullptr, nullptr, none, EscSel{nullptr, 0, 0u}, tile_ws, nullptr,
                       nlaunch);
    if (e != cudaSuccess) return e;
  }
  k_splits<<<(nparts + 1 + 255) / 256, 256, 0, s>>>(m, nprod_scan, nparts, splits_dev);
  if (nlaunch) *nlaunch += 2;
  return cudaGetLastError();
}

}  // namespace spg
