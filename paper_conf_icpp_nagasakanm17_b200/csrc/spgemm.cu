// spgemm.cu — C ABI (include/spgemm.h) and host orchestration of the two-phase hash SpGEMM
// (Figure 1 steps (1)-(7)) on one B200.
//
//   spgemm_symbolic:  (1)+(2) k_nprod_group  -> [sync 1: group sizes, max n_prod]
//                     (2) k_group_scatter
//                     (3) per-group hash-count kernels, one stream per group,
//                         optimistic group -> global retry on the same stream
//                     (4) tile scan into rpt_C, fused with (6)'s grouping by nnz
//                     -> [sync 2: nnz(C)] (the host must allocate C exactly)
//   spgemm_numeric:   (6) k_group_scatter by nnz, (7) per-group accumulate/gather/sort kernels,
//                     one stream per group; asynchronous.
#include <cuda_runtime.h>

#include <algorithm>
#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <string>
#include <vector>

#include "spgemm.h"
#include "spgemm_internal.cuh"

using namespace spg;

namespace {

constexpr int kNumStreams = 8;

struct Buf {
  void* p = nullptr;
  size_t bytes = 0;
};

struct GraphEntry {
  cudaGraphExec_t exec = nullptr;
  std::vector<long long> key;    // full key: topology + every pointer the kernels see
  std::vector<long long> topo;   // topology key: launch structure only (grids, groups, options)
  int launches = 0;              // kernels in the captured segment
  bool timed[16] = {};           // groups with timing events in the segment
  int kind[16] = {};             // spgemm_kernel_t of every group in the segment
};
// The active (most recent) entry plus up to kGraphSpare others, most recent first: callers that
// alternate output buffers (a caching allocator hands back two or three addresses in turn) replay
// an instantiated graph instead of re-capturing and updating one every call.
constexpr size_t kGraphSpare = 3;
struct GraphCache : GraphEntry {
  std::vector<GraphEntry> others;
  void destroy() {
    if (exec) cudaGraphExecDestroy(exec);
    exec = nullptr;
    for (GraphEntry& e : others)
      if (e.exec) cudaGraphExecDestroy(e.exec);
    others.clear();
  }
};

struct DeviceGuard {
  int prev = -1;
  explicit DeviceGuard(int d) {
    if (cudaGetDevice(&prev) == cudaSuccess && prev != d) cudaSetDevice(d);
  }
  ~DeviceGuard() {
    int cur;
    if (prev >= 0 && cudaGetDevice(&cur) == cudaSuccess && cur != prev) cudaSetDevice(prev);
  }
};

long long next_pow2(long long x) {
  long long p = 1;
  while (p < x) p <<= 1;
  return p;
}

}  // namespace

struct spgemm_ctx {
  int device = 0;
  int num_sms = 148;
  cudaStream_t stream = nullptr;   // internal execution stream (capturable, non-blocking)
  cudaStream_t ustream = nullptr;  // the caller's stream given to spgemm_create
  cudaEvent_t ev_enter = nullptr, ev_leave = nullptr;
  spgemm_allocator_t alloc{};
  bool user_alloc = false;
  cudaMemPool_t pool = nullptr;  // private stream-ordered pool; memory retained across calls
  cudaStream_t gs[kNumStreams]{};
  cudaEvent_t fork_ev = nullptr;
  cudaEvent_t join_ev[kNumStreams]{};
  cudaEvent_t ev[8]{};
  cudaEvent_t gstart[2][kMaxGroups]{}, gstop[2][kMaxGroups]{};
  bool gtimed[2][kMaxGroups]{};
  int gkind[2][kMaxGroups]{};    // spgemm_kernel_t per group of the last call (stats)
  bool gtimed_phases = false;  // ev[1], ev[2] recorded (per-group events on)
  // options
  int sym_min_group = -1, num_min_group = -1, fill_limit = 0, use_streams = 1, validate = 0, lanes = 0;
  int long_len = 0;  // 0 auto, -1 off
  int range_hash = 1;  // 1: range-offset hash where a row's column span fits
  int cluster_fill = 0;  // symbolic cluster table fill limit (0 = capacity / 2)
  int use_cluster = 1;   // 0: rows beyond one CTA go straight to global memory (ablation)
  int flat = -1;         // load-balanced flattened product loop: -1 auto (mean B row < 16), 0, 1
  int timing = 1;
  int range_warp = 1;    // warp-per-row kernels for range rows (kernels_range.cu)
  long long range_min_np = kRangeMinNprodDefault;
  int rank_acc = 1;      // CTA-per-row groups: rank-indexed tables (kernels_rankacc.cu)
  // rank kernels only for groups with 100 * level-1 words <= pct * group key bound (0: always);
  // R-MAT s22 (4097 words), rank vs paper hash + bucket sort: numeric group 4 (bound 256) 11.6 vs
  // 4.1 ms, group 5 (512) 13.5 vs 9.0, group 6 (1024) 14.6 vs 17.8; symbolic group 6 (2048) 6.7
  // vs 4.5, group 7 (4096) 3.6 vs 4.6
  // (symbolic 100 since the multiplicative hash's top-bit slots: R-MAT s22 symbolic group 7 hash 2.94 vs
  // rank count 3.33 ms; s20 group 5 0.71 vs 0.73; other configs unchanged)
  long long rank_l1_pct = 500, rank_l1_pct_sym = 100;
  int tiny = 1;          // groups 0-1: thread-per-row register tables (kernels_tiny.cu)
  int small_opt = 1;     // small matrices (m <= kSmallRows): one-launch phases, no grouping (kernels_tiny.cu)
  // warp-per-row register sort (kernels_wsort.cu): bit 1 symbolic, bit 2 numeric.  Off by default:
  // measured 2.5-9x slower than the hash / ESC kernels on every graph config (R-MAT s16-s22, webbase,
  // Economics, Circuit; scripts/ab.py): the unrolled networks' register footprint (up to 240 per
  // thread) leaves 8-16 warps per SM and the shuffle stages serialise
  int wsort = 0;
  // symbolic optimistic-group rows counted exactly by the chunked rank-count kernel (R-MAT s22:
  // 1811 rows with n_prod_i > 16384)
  int rank_big_sym = 1;
  int rank_big_shared = 1;
  // numeric group 9: 2 = products in registers, output reduced into C, two 512-thread CTAs per SM
  // (R-MAT s22 6.87 -> 5.54 ms); 1 = persistent rank-big kernel with level 2 in shared memory
  // (6.32 ms); 0 = one 1024-thread CTA per row, the row in shared memory
  int rank_mid = 2;
  int rank_gout = 0;
  int rank_big_max = 3;  // numeric big groups 10..10+rank_big_max-1 on the rank-big kernel, the rest on clusters  // numeric rank groups 3-8 with the output reduced into C (no vals/keys arrays)  // numeric group 10 rank-big rows: level 2 in shared memory (if it fits)
  bool small = false;    // the last symbolic call took the small-matrix path
  std::vector<long long> small_miss;  // inputs whose last small-path attempt overflowed (skip it)
  // batched graph-row kernels (kernels_esc.cu): bit 1 symbolic groups 2-9 (off by default: R-MAT s22
  // 26.5 ms vs 21.7 ms with the per-group hash / rank-count kernels), bit 2 numeric ESC
  int batch = 2;
  long long esc_pct = 200;  // numeric ESC rows: 100 * n_prod_i <= esc_pct * nnz_i
  long long esc_mask = -1;  // symbolic groups whose rows may take the numeric ESC kernels (-1: auto)
  long long esc_w_pct = 100;  // auto rule: ESC where 100 * (n/1024 + 1) >= esc_w_pct * group bound
  bool phase_streams = true;  // the current phase forks per-group streams (phase_concurrent)
  // CTA-per-row numeric hash groups: two-level bitmap rank (else bucket sort); 1 = only where the
  // level-1 width W <= the group's nnz bound (R-MAT s22, W = 4097: bucket 4.1 ms vs bitmap 21.9 ms
  // on group 4, 25.4 vs 28.5 on group 7), 2 = always
  int bitmap_rank = 1;
  long long ws_budget = 8LL << 30;
  // state of the last symbolic call
  int state = 0;
  bool numeric_done = false;
  long long m = 0, k = 0, n = 0, nnza = 0, nnzb = 0, nnzc = 0;
  const int64_t *a_rpt = nullptr, *b_rpt = nullptr;
  const int32_t *a_col = nullptr, *b_col = nullptr;
  int64_t* c_rpt = nullptr;
  int vw_log2 = 0;
  Buf defer_b;  // step (1): deferred long B rows (the A list reuses perm1, rewritten after sync 1)
  Buf binfo;  // step (1): {min col, max col, length} of every B row (one 16-byte gather per A entry)
  Buf nprod, grp1, grp2, perm1, perm2, acc, tiles, overflow, overflow2, slab_sym, bmm, rlohi, num_slab, num_slab_c,
      rbits, bbits;
  bool range_num = false;  // numeric range rows on for the last symbolic call (bitmap allocated, B sorted)
  GraphCache gsym, gnum;  // captured segments (see run_graph)
  GraphCache gsmall;      // small-matrix symbolic segment
  int use_graphs = 1;
  bool perm2_ready = false;
  bool group_sums_done = false;  // per-group n_prod/nnz sums (computed on demand by get_stats)
  DevAcc* hacc = nullptr;      // pinned
  DevAcc* hacc_dev = nullptr;  // the same memory as a device pointer (mapped pinned memory)
  long long* hends = nullptr;  // pinned: a_rpt[0], a_rpt[m], b_rpt[0], b_rpt[k]
  DevAcc snap1{}, snap2{};
  spgemm_stats_t stats{};
  long long ws_cur = 0, ws_peak = 0;
  std::string err;
};

namespace {

spgemm_status_t fail(spgemm_handle_t h, spgemm_status_t s, const std::string& msg) {
  if (h) h->err = msg;
  return s;
}

spgemm_status_t fail_cuda(spgemm_handle_t h, cudaError_t e, const char* what) {
  char buf[512];
  snprintf(buf, sizeof buf, "%s: %s (%s)", what, cudaGetErrorName(e), cudaGetErrorString(e));
  return fail(h, SPGEMM_ERR_CUDA, buf);
}

#define CK(x)                                                  \
  do {                                                         \
    cudaError_t e_ = (x);                                      \
    if (e_ != cudaSuccess) return fail_cuda(h, e_, #x);        \
  } while (0)

spgemm_status_t buf_alloc(spgemm_handle_t h, Buf& b, size_t bytes) {
  b.p = nullptr;
  b.bytes = 0;
  if (bytes == 0) return SPGEMM_OK;
  bytes = (bytes + 255) & ~size_t(255);
  if (h->user_alloc) {
    b.p = h->alloc.alloc(bytes, (void*)h->stream, h->alloc.ctx);
    if (!b.p) return fail(h, SPGEMM_ERR_OOM, "allocator returned NULL for " + std::to_string(bytes) + " bytes");
  } else {
    cudaError_t e = cudaMallocFromPoolAsync(&b.p, bytes, h->pool, h->stream);
    if (e != cudaSuccess) {
      cudaGetLastError();
      b.p = nullptr;
      return fail(h, SPGEMM_ERR_OOM, std::string("cudaMallocFromPoolAsync: ") + cudaGetErrorString(e));
    }
  }
  b.bytes = bytes;
  h->ws_cur += (long long)bytes;
  h->ws_peak = std::max(h->ws_peak, h->ws_cur);
  return SPGEMM_OK;
}

void buf_free(spgemm_handle_t h, Buf& b) {
  if (!b.p) return;
  if (h->user_alloc) h->alloc.free(b.p, b.bytes, (void*)h->stream, h->alloc.ctx);
  else cudaFreeAsync(b.p, h->stream);
  h->ws_cur -= (long long)b.bytes;
  b.p = nullptr;
  b.bytes = 0;
}

// Grow-only workspace: buffers are kept across calls (stable addresses let the captured CUDA
// graphs replay) and grown when a call needs more; spgemm_destroy releases them.
spgemm_status_t buf_ensure(spgemm_handle_t h, Buf& b, size_t bytes) {
  if (bytes == 0) return SPGEMM_OK;
  if (b.p && b.bytes >= ((bytes + 255) & ~size_t(255))) return SPGEMM_OK;
  buf_free(h, b);
  return buf_alloc(h, b, bytes);
}

void release_state(spgemm_handle_t h) {
  h->state = 0;
  h->perm2_ready = false;
}

void free_all(spgemm_handle_t h) {
  Buf* all[] = {&h->nprod, &h->grp1, &h->grp2, &h->perm1, &h->perm2, &h->acc, &h->tiles, &h->overflow,
                &h->overflow2, &h->slab_sym, &h->bmm, &h->rlohi, &h->num_slab, &h->num_slab_c, &h->rbits, &h->bbits,
                &h->binfo,
                &h->defer_b};
  for (Buf* b : all) buf_free(h, *b);
  release_state(h);
}

// Capture `enqueue` (async work on h->stream and the forked group streams) into a CUDA graph the
// first time `topo` is seen and replay it while topology and pointers are unchanged; when only the
// pointers differ (new output buffers, new inputs of the same structure) the capture is re-run and
// applied to the instantiated graph with cudaGraphExecUpdate instead of a fresh instantiate (per-group launches on 8
// streams become one graph launch; the paper's concurrent per-group kernels).
bool graphs_on(spgemm_handle_t h) { return h->use_graphs && h->timing < 2; }
// per-group kernel events are recorded only outside graphs (events inside a graph cannot time)
bool group_events(spgemm_handle_t h) { return h->timing >= 2 || (h->timing == 1 && !h->use_graphs); }

template <typename Fn>
spgemm_status_t run_graph(spgemm_handle_t h, GraphCache& gc, const std::vector<long long>& topo,
                          const std::vector<long long>& ptrs, Fn&& enqueue) {
  if (!graphs_on(h)) return enqueue();
  std::vector<long long> key = topo;
  key.insert(key.end(), ptrs.begin(), ptrs.end());
  if (!(gc.exec && gc.key == key)) {  // an older entry of the same call becomes the active one
    for (size_t i = 0; i < gc.others.size(); ++i)
      if (gc.others[i].exec && gc.others[i].key == key) {
        GraphEntry hit = std::move(gc.others[i]);
        gc.others.erase(gc.others.begin() + (long)i);
        gc.others.insert(gc.others.begin(), std::move(static_cast<GraphEntry&>(gc)));
        static_cast<GraphEntry&>(gc) = std::move(hit);
        break;
      }
  }
  if (gc.exec && gc.key == key) {  // identical call: replay
    CK(cudaGraphLaunch(gc.exec, h->stream));
    ++h->stats.graph_replays;
    return SPGEMM_OK;
  }
  // a new call: keep the active entry while there is room, else recycle the least recently used
  // entry (updated in place when its topology matches, else re-instantiated)
  if (gc.exec) {
    gc.others.insert(gc.others.begin(), std::move(static_cast<GraphEntry&>(gc)));
    static_cast<GraphEntry&>(gc) = GraphEntry{};
    if (gc.others.size() > kGraphSpare) {
      size_t v = gc.others.size() - 1;  // LRU, or the least recent one with the same topology
      for (size_t i = gc.others.size(); i-- > 0;)
        if (gc.others[i].topo == topo) { v = i; break; }
      static_cast<GraphEntry&>(gc) = std::move(gc.others[v]);
      gc.others.erase(gc.others.begin() + (long)v);
    }
  }
  cudaGraph_t g = nullptr;
  CK(cudaStreamBeginCapture(h->stream, cudaStreamCaptureModeThreadLocal));
  const spgemm_status_t s = enqueue();
  cudaError_t e = cudaStreamEndCapture(h->stream, &g);
  if (s != SPGEMM_OK) {
    if (g) cudaGraphDestroy(g);
    cudaGetLastError();
    return s;
  }
  if (e != cudaSuccess) return fail_cuda(h, e, "cudaStreamEndCapture");
  bool updated = false;
  if (gc.exec && gc.topo == topo) {  // same launch structure, new buffers: update the kernel params in place
    cudaGraphExecUpdateResultInfo info{};
    updated = cudaGraphExecUpdate(gc.exec, g, &info) == cudaSuccess;
    if (!updated) cudaGetLastError();
    else ++h->stats.graph_replays;
  }
  if (!updated) {
    if (gc.exec) {
      cudaGraphExecDestroy(gc.exec);
      gc.exec = nullptr;
    }
    e = cudaGraphInstantiate(&gc.exec, g, 0);
    if (e != cudaSuccess) {
      cudaGraphDestroy(g);
      gc.exec = nullptr;
      return fail_cuda(h, e, "cudaGraphInstantiate");
    }
  }
  cudaGraphDestroy(g);
  gc.key = key;
  gc.topo = topo;
  CK(cudaGraphLaunch(gc.exec, h->stream));
  return SPGEMM_OK;
}

#define ALLOC(buf, bytes)                                          \
  do {                                                             \
    spgemm_status_t s_ = buf_ensure(h, (buf), (bytes));            \
    if (s_ != SPGEMM_OK) return s_;                                \
  } while (0)

// Range rows (kernels_range.cu) need the column spans (range hash on) and are not used when a
// minimum group is forced (the forced-path tests pin every hash-table group).
bool sym_range_on(spgemm_handle_t h) { return h->range_warp && h->range_hash && h->sym_min_group < 0; }

Bounds sym_bounds(spgemm_handle_t h) {
  Bounds b{};
  for (int i = 0; i < kNumSymBounds; ++i) b.upper[i] = kSymGroups[i].upper;
  b.nbounds = kNumSymBounds;
  b.min_group = h->sym_min_group;
  b.range_group = sym_range_on(h) ? kSymRange : -1;
  b.range_min_np = h->range_min_np;
  b.range_k = h->k;
  return b;
}

// Numeric range rows: the phase-1 range rows, when every B row is strictly increasing (plain
// read-modify-write accumulation), the pattern bitmap fits the workspace budget and no numeric
// group is forced (decided at sync 1: h->range_num).
Bounds num_bounds(spgemm_handle_t h) {
  Bounds b{};
  for (int i = 0; i < kNumNumBounds; ++i) b.upper[i] = kNumGroups[i].upper;
  b.nbounds = kNumNumBounds;
  b.min_group = h->num_min_group;
  b.range_group = h->range_num ? kNumRange : -1;
  b.range_min_np = 0;
  return b;
}

Offsets offsets_of(const unsigned long long* rows, int ngroups) {
  Offsets o{};
  o.ngroups = ngroups;
  long long run = 0;
  for (int g = 0; g < ngroups; ++g) {
    o.off[g] = run;
    run += (long long)rows[g];
  }
  o.off[ngroups] = run;
  return o;
}

// Order the internal stream after the caller's stream (entry) and the caller's stream after the
// internal one (exit).
cudaError_t enter(spgemm_handle_t h) {
  cudaError_t e = cudaEventRecord(h->ev_enter, h->ustream);
  return e == cudaSuccess ? cudaStreamWaitEvent(h->stream, h->ev_enter, 0) : e;
}
cudaError_t leave(spgemm_handle_t h) {
  cudaError_t e = cudaEventRecord(h->ev_leave, h->stream);
  return e == cudaSuccess ? cudaStreamWaitEvent(h->ustream, h->ev_leave, 0) : e;
}

// Per-group streams only when the phase has >= 2 non-empty groups (one group: the fork/join
// events cost ~3 % of the cant step for nothing).
bool phase_concurrent(spgemm_handle_t h, const unsigned long long* rows, int ngroups) {
  int ne = 0;
  for (int g = 0; g < ngroups; ++g) ne += rows[g] > 0;
  return h->use_streams && ne >= 2;
}
cudaStream_t group_stream(spgemm_handle_t h, int g) { return h->phase_streams ? h->gs[g % kNumStreams] : h->stream; }

cudaError_t fork(spgemm_handle_t h) {
  if (!h->phase_streams) return cudaSuccess;
  cudaError_t e = cudaEventRecord(h->fork_ev, h->stream);
  for (int i = 0; i < kNumStreams && e == cudaSuccess; ++i) e = cudaStreamWaitEvent(h->gs[i], h->fork_ev, 0);
  return e;
}

cudaError_t join(spgemm_handle_t h) {
  if (!h->phase_streams) return cudaSuccess;
  cudaError_t e = cudaSuccess;
  for (int i = 0; i < kNumStreams && e == cudaSuccess; ++i) {
    e = cudaEventRecord(h->join_ev[i], h->gs[i]);
    if (e == cudaSuccess) e = cudaStreamWaitEvent(h->stream, h->join_ev[i], 0);
  }
  return e;
}

int auto_vw_log2(spgemm_handle_t h) {
  if (h->lanes > 0) {
    int l = 0;
    while ((1 << (l + 1)) <= h->lanes && l < 5) ++l;
    return l;
  }
  const double avg = h->k > 0 ? (double)h->nnzb / (double)h->k : 1.0;
  if (avg >= 24.0) {  // widest sub-group that wastes <= 10 % of its lanes on a mean-length B row
    for (int l = 5; l >= 3; --l) {  // (QCD-like, 39 per row: 8 lanes, not 32 — measured 4 lanes 129 vs 32 lanes 118 GFLOPS)
      const double w = (double)(1 << l);
      if (std::ceil(avg / w) * w <= 1.1 * avg) return l;
    }
    return 3;
  }
  int l = 0;
  while (l < 5 && (double)(1 << (l + 1)) <= avg * 1.5) ++l;
  return l;
}

// CTA-per-row kernels hand B rows longer than this to the whole CTA (load balance).
bool flat_of(spgemm_handle_t h) {
  if (h->flat >= 0) return h->flat != 0;
  return h->k > 0 && (double)h->nnzb / (double)h->k < 16.0;
}

// Symbolic groups whose weakly compressing rows take the numeric ESC kernels (kernels_esc.cu)
// instead of the rank-indexed CTA-per-row kernels, whose level-1 bitmap costs W = n/1024 + 1 words
// per row whatever the row's size: ESC where 100 * W >= esc_w_pct * B (B = the group's n_prod
// bound).  Measured per group (scripts/esc_groups.py, serial, fp32, ESC at 48 warps per SM):
// R-MAT s22 (W = 4097) ESC saves 1.9 / 2.0 / 4.8 / 7.8 / 4.2 / 0.8 ms on groups 2-7 (W/B = 32 ..
// 1) and breaks even on group 8 (W/B = 0.5); R-MAT s20 (W = 1025) saves 0.46 / 0.26 / 0.10 /
// 0.08 ms on groups 2-5 (W/B = 8 .. 1), loses 0.23 ms on group 6 (W/B = 0.5); webbase, R-MAT
// s16/s18, Economics, Circuit lose on most groups (W <= 1024: their level-1 bitmaps are cheap;
// webbase's 95 %-local rows also skew the buckets, which costs the ESC kernels a refinement pass).
unsigned esc_auto_mask(spgemm_handle_t h) {
  const long long W = h->n / 1024 + 1;
  unsigned m = 0;
  if (h->wsort & 2)  // warp-sorted rows (kernels_wsort.cu): groups 2..wsort_max_group() on any matrix
    for (int g = kEscSymLo; g <= wsort_max_group(); ++g) m |= 1u << g;
  for (int g = kEscSymLo; g <= kEscSymHi; ++g)
    if (100 * W >= h->esc_w_pct * kSymGroups[g].upper && W > 1024) m |= 1u << g;
  return m;
}

int long_len_of(spgemm_handle_t h) {
  if (h->long_len < 0) return 0;
  if (h->long_len > 0) return h->long_len;
  return std::max(64, 8 << h->vw_log2);
}

}  // namespace

extern "C" {

const char* spgemm_version(void) { return "spgemm-b200 sm_100a (" __DATE__ ")"; }

const char* spgemm_status_string(spgemm_status_t s) {
  switch (s) {
    case SPGEMM_OK: return "SPGEMM_OK";
    case SPGEMM_ERR_INVALID_ARG: return "SPGEMM_ERR_INVALID_ARG";
    case SPGEMM_ERR_BAD_STATE: return "SPGEMM_ERR_BAD_STATE";
    case SPGEMM_ERR_OOM: return "SPGEMM_ERR_OOM";
    case SPGEMM_ERR_CUDA: return "SPGEMM_ERR_CUDA";
    case SPGEMM_ERR_INDEX_OVERFLOW: return "SPGEMM_ERR_INDEX_OVERFLOW";
    case SPGEMM_ERR_NOT_SUPPORTED: return "SPGEMM_ERR_NOT_SUPPORTED";
    case SPGEMM_ERR_INVALID_INPUT: return "SPGEMM_ERR_INVALID_INPUT";
  }
  return "SPGEMM_ERR_UNKNOWN";
}

const char* spgemm_last_error(spgemm_handle_t h) { return h ? h->err.c_str() : "null handle"; }

spgemm_status_t spgemm_group_bounds(int phase, int64_t* upper, int32_t* ngroups) {
  if (!upper || !ngroups || (phase != 1 && phase != 2)) return SPGEMM_ERR_INVALID_ARG;
  if (phase == 1) {
    for (int i = 0; i < kNumSymBounds; ++i) upper[i] = kSymGroups[i].upper;
    *ngroups = kNumSymBounds;
  } else {
    for (int i = 0; i < kNumNumBounds; ++i) upper[i] = kNumGroups[i].upper;
    *ngroups = kNumNumBounds;
  }
  return SPGEMM_OK;
}

spgemm_status_t spgemm_create(spgemm_handle_t* out, int device, void* stream, const spgemm_allocator_t* alloc) {
  if (!out) return SPGEMM_ERR_INVALID_ARG;
  *out = nullptr;
  if (alloc && (!alloc->alloc || !alloc->free)) return SPGEMM_ERR_INVALID_ARG;
  spgemm_ctx* h = new spgemm_ctx();
  h->device = device;
  h->ustream = (cudaStream_t)stream;
  if (alloc) {
    h->alloc = *alloc;
    h->user_alloc = true;
  }
  cudaDeviceProp prop;
  cudaError_t e = cudaGetDeviceProperties(&prop, device);
  if (e != cudaSuccess) {
    spgemm_status_t s = fail_cuda(h, e, "cudaGetDeviceProperties");
    *out = h;  // keep the handle so spgemm_last_error works; caller destroys it
    return s;
  }
  if (prop.major != 10) {
    *out = h;
    return fail(h, SPGEMM_ERR_NOT_SUPPORTED, std::string("device is not sm_100 (B200): ") + prop.name);
  }
  h->num_sms = prop.multiProcessorCount;
  DeviceGuard g(device);
  for (int i = 0; i < kNumStreams; ++i) {
    e = cudaStreamCreateWithFlags(&h->gs[i], cudaStreamNonBlocking);
    if (e == cudaSuccess) e = cudaEventCreateWithFlags(&h->join_ev[i], cudaEventDisableTiming);
    if (e != cudaSuccess) break;
  }
  if (e == cudaSuccess) e = cudaEventCreateWithFlags(&h->fork_ev, cudaEventDisableTiming);
  // all work runs on an internal stream joined to the caller's stream at every entry/exit (the
  // legacy default stream cannot be captured into a CUDA graph)
  if (e == cudaSuccess) e = cudaStreamCreateWithFlags(&h->stream, cudaStreamNonBlocking);
  if (e == cudaSuccess) e = cudaEventCreateWithFlags(&h->ev_enter, cudaEventDisableTiming);
  if (e == cudaSuccess) e = cudaEventCreateWithFlags(&h->ev_leave, cudaEventDisableTiming);
  for (int i = 0; i < 8 && e == cudaSuccess; ++i) e = cudaEventCreate(&h->ev[i]);
  for (int p = 0; p < 2; ++p)
    for (int i = 0; i < kMaxGroups && e == cudaSuccess; ++i) {
      e = cudaEventCreate(&h->gstart[p][i]);
      if (e == cudaSuccess) e = cudaEventCreate(&h->gstop[p][i]);
    }
  if (e == cudaSuccess && !h->user_alloc) {
    // Private pool whose memory stays mapped between calls (release threshold = max): the
    // default pool unmaps at every synchronisation, which re-maps the global-memory hash
    // slabs (up to hundreds of MB) on every call.  Trimmed in spgemm_destroy.
    cudaMemPoolProps props{};
    props.allocType = cudaMemAllocationTypePinned;
    props.location.type = cudaMemLocationTypeDevice;
    props.location.id = device;
    e = cudaMemPoolCreate(&h->pool, &props);
    if (e == cudaSuccess) {
      unsigned long long thr = ~0ull;
      e = cudaMemPoolSetAttribute(h->pool, cudaMemPoolAttrReleaseThreshold, &thr);
    }
  }
  if (e == cudaSuccess) e = cudaMallocHost(&h->hacc, sizeof(DevAcc));
  if (e == cudaSuccess) e = cudaHostGetDevicePointer(reinterpret_cast<void**>(&h->hacc_dev), h->hacc, 0);
  if (e == cudaSuccess) e = cudaMallocHost(&h->hends, 4 * sizeof(long long));
  *out = h;
  if (e != cudaSuccess) return fail_cuda(h, e, "spgemm_create");
  return SPGEMM_OK;
}

spgemm_status_t spgemm_destroy(spgemm_handle_t h) {
  if (!h) return SPGEMM_ERR_INVALID_ARG;
  {
    DeviceGuard g(h->device);
    if (h->hacc) {  // hacc is allocated only on a supported device
      free_all(h);
      cudaStreamSynchronize(h->stream);
    }
    h->gsym.destroy();
    h->gnum.destroy();
    h->gsmall.destroy();
    for (int i = 0; i < kNumStreams; ++i) {
      if (h->gs[i]) cudaStreamDestroy(h->gs[i]);
      if (h->join_ev[i]) cudaEventDestroy(h->join_ev[i]);
    }
    if (h->fork_ev) cudaEventDestroy(h->fork_ev);
    if (h->ev_enter) cudaEventDestroy(h->ev_enter);
    if (h->ev_leave) cudaEventDestroy(h->ev_leave);
    if (h->stream) cudaStreamDestroy(h->stream);
    for (auto& e : h->ev) if (e) cudaEventDestroy(e);
    for (int p = 0; p < 2; ++p)
      for (int i = 0; i < kMaxGroups; ++i) {
        if (h->gstart[p][i]) cudaEventDestroy(h->gstart[p][i]);
        if (h->gstop[p][i]) cudaEventDestroy(h->gstop[p][i]);
      }
    if (h->hacc) cudaFreeHost(h->hacc);
    if (h->hends) cudaFreeHost(h->hends);
    if (h->pool) {
      cudaMemPoolTrimTo(h->pool, 0);
      cudaMemPoolDestroy(h->pool);
    }
  }
  delete h;
  return SPGEMM_OK;
}

spgemm_status_t spgemm_set_option(spgemm_handle_t h, spgemm_option_t opt, int64_t v) {
  if (!h) return SPGEMM_ERR_INVALID_ARG;
  switch (opt) {
    case SPGEMM_OPT_SYM_MIN_GROUP:
      if (v < -1 || v > kSymGlobal) return fail(h, SPGEMM_ERR_INVALID_ARG, "SYM_MIN_GROUP out of range");
      h->sym_min_group = (int)v; break;
    case SPGEMM_OPT_NUM_MIN_GROUP:
      if (v < -1 || v > kNumGlobal) return fail(h, SPGEMM_ERR_INVALID_ARG, "NUM_MIN_GROUP out of range");
      h->num_min_group = (int)v; break;
    case SPGEMM_OPT_SYM_FILL_LIMIT:
      if (v < 0) return fail(h, SPGEMM_ERR_INVALID_ARG, "FILL_LIMIT < 0");
      h->fill_limit = (int)std::min<int64_t>(v, 1 << 30); break;
    case SPGEMM_OPT_STREAMS: h->use_streams = v ? 1 : 0; break;
    case SPGEMM_OPT_VALIDATE: h->validate = v ? 1 : 0; break;
    case SPGEMM_OPT_LANES:
      if (v < 0 || v > 32 || (v & (v - 1))) return fail(h, SPGEMM_ERR_INVALID_ARG, "LANES must be 0 or a power of two <= 32");
      h->lanes = (int)v; break;
    case SPGEMM_OPT_WORKSPACE_BUDGET:
      if (v <= 0) return fail(h, SPGEMM_ERR_INVALID_ARG, "budget must be > 0");
      h->ws_budget = v; break;
    case SPGEMM_OPT_TIMING:
      if (v < 0 || v > 2) return fail(h, SPGEMM_ERR_INVALID_ARG, "TIMING must be 0, 1 or 2");
      h->timing = (int)v; break;
    case SPGEMM_OPT_RANGE_HASH: h->range_hash = v ? 1 : 0; break;
    case SPGEMM_OPT_CLUSTER: h->use_cluster = v ? 1 : 0; break;
    case SPGEMM_OPT_GRAPHS: h->use_graphs = v ? 1 : 0; break;
    case SPGEMM_OPT_FLAT:
      if (v < -1 || v > 1) return fail(h, SPGEMM_ERR_INVALID_ARG, "FLAT must be -1, 0 or 1");
      h->flat = (int)v; break;
    case SPGEMM_OPT_CLUSTER_FILL_LIMIT:
      if (v < 0) return fail(h, SPGEMM_ERR_INVALID_ARG, "CLUSTER_FILL_LIMIT < 0");
      h->cluster_fill = (int)std::min<int64_t>(v, 1 << 30); break;
    case SPGEMM_OPT_RANGE_WARP:
      if (v < 0 || v > 2) return fail(h, SPGEMM_ERR_INVALID_ARG, "RANGE_WARP must be 0, 1 or 2");
      h->range_warp = (int)v; break;
    case SPGEMM_OPT_RANGE_MIN_NPROD:
      if (v < 1 || v > kRangeMaxNprod) return fail(h, SPGEMM_ERR_INVALID_ARG, "RANGE_MIN_NPROD out of range");
      h->range_min_np = v; break;
    case SPGEMM_OPT_BITMAP_RANK:
      if (v < 0 || v > 2) return fail(h, SPGEMM_ERR_INVALID_ARG, "BITMAP_RANK must be 0, 1 or 2");
      h->bitmap_rank = (int)v; break;
    case SPGEMM_OPT_RANK_ACC: h->rank_acc = v ? 1 : 0; break;
    case SPGEMM_OPT_RANK_L1_PCT:
      if (v < 0 || v > (1LL << 40)) return fail(h, SPGEMM_ERR_INVALID_ARG, "RANK_L1_PCT out of range");
      h->rank_l1_pct = v; break;
    case SPGEMM_OPT_RANK_L1_PCT_SYM:
      if (v < 0 || v > (1LL << 40)) return fail(h, SPGEMM_ERR_INVALID_ARG, "RANK_L1_PCT_SYM out of range");
      h->rank_l1_pct_sym = v; break;
    case SPGEMM_OPT_TINY:
      if (v < 0 || v > 2) return fail(h, SPGEMM_ERR_INVALID_ARG, "TINY must be 0, 1 or 2");
      h->tiny = (int)v; break;
    case SPGEMM_OPT_BATCH:
      if (v < 0 || v > 3) return fail(h, SPGEMM_ERR_INVALID_ARG, "BATCH must be 0..3");
      h->batch = (int)v; break;
    case SPGEMM_OPT_ESC_PCT:
      if (v < 0 || v > (1LL << 40)) return fail(h, SPGEMM_ERR_INVALID_ARG, "ESC_PCT out of range");
      h->esc_pct = v; break;
    case SPGEMM_OPT_ESC_GROUPS: h->esc_mask = v; break;
    case SPGEMM_OPT_SMALL: h->small_opt = v ? 1 : 0; break;
    case SPGEMM_OPT_RANK_BIG_SHARED:
      if (v < 0 || v > 2) return fail(h, SPGEMM_ERR_INVALID_ARG, "RANK_BIG_SHARED must be 0, 1 or 2");
      h->rank_big_shared = (int)v; break;
    case SPGEMM_OPT_RANK_GOUT: h->rank_gout = v ? 1 : 0; break;
    case SPGEMM_OPT_RANK_BIG_MAX:
      if (v < 0 || v > 3) return fail(h, SPGEMM_ERR_INVALID_ARG, "RANK_BIG_MAX must be 0..3");
      h->rank_big_max = (int)v; break;
    case SPGEMM_OPT_RANK_MID:
      if (v < 0 || v > 2) return fail(h, SPGEMM_ERR_INVALID_ARG, "RANK_MID must be 0, 1 or 2");
      h->rank_mid = (int)v; break;
    case SPGEMM_OPT_RANK_BIG_SYM:
      if (v < 0 || v > 2) return fail(h, SPGEMM_ERR_INVALID_ARG, "RANK_BIG_SYM must be 0, 1 or 2");
      h->rank_big_sym = (int)v; break;
    case SPGEMM_OPT_WSORT:
      if (v < 0 || v > 3) return fail(h, SPGEMM_ERR_INVALID_ARG, "WSORT must be 0..3");
      h->wsort = (int)v; break;
    case SPGEMM_OPT_LONG_ROW:
      if (v < -1 || v > (1 << 30)) return fail(h, SPGEMM_ERR_INVALID_ARG, "LONG_ROW out of range");
      h->long_len = (int)v; break;
    default: return fail(h, SPGEMM_ERR_INVALID_ARG, "unknown option");
  }
  return SPGEMM_OK;
}

spgemm_status_t spgemm_symbolic(spgemm_handle_t h, int64_t m, int64_t k, int64_t n, const int64_t* a_rpt,
                                const int32_t* a_col, const int64_t* b_rpt, const int32_t* b_col,
                                int64_t* c_rpt, int64_t* c_nnz, int64_t* nprod_out) {
  if (!h) return SPGEMM_ERR_INVALID_ARG;
  if (!h->hacc) return fail(h, SPGEMM_ERR_BAD_STATE, "handle was not created successfully");
  if (m < 0 || k < 0 || n < 0) return fail(h, SPGEMM_ERR_INVALID_ARG, "negative dimension");
  if (!a_rpt || !b_rpt || !c_rpt || !c_nnz) return fail(h, SPGEMM_ERR_INVALID_ARG, "NULL pointer argument");
  if (n > 2147483646LL || m >= 2147483647LL || k >= 2147483647LL)
    return fail(h, SPGEMM_ERR_INDEX_OVERFLOW, "dimensions exceed int32 column/row indices");
  DeviceGuard dg(h->device);
  CK(enter(h));
  release_state(h);
  h->numeric_done = false;
  h->m = m; h->k = k; h->n = n;
  h->a_rpt = a_rpt; h->a_col = a_col; h->b_rpt = b_rpt; h->b_col = b_col; h->c_rpt = c_rpt;
  memset(&h->stats, 0, sizeof h->stats);
  memset(h->gtimed, 0, sizeof h->gtimed);
  memset(h->gkind, 0, sizeof h->gkind);
  h->ws_peak = h->ws_cur;
  h->stats.m = m; h->stats.k = k; h->stats.n = n;
  h->stats.n_sym_groups = kNumSymGroups;
  h->stats.n_num_groups = kNumNumGroups;
  long long launches = 0;

  ALLOC(h->acc, sizeof(DevAcc));
  DevAcc* dacc = static_cast<DevAcc*>(h->acc.p);
  const std::vector<long long> small_key = {m, k, n, (long long)a_rpt, (long long)a_col, (long long)b_rpt,
                                             (long long)b_col};
  const bool small_try = h->small_opt && m > 0 && m <= kSmallRows && h->sym_min_group < 0 && h->num_min_group < 0 &&
                         h->tiny >= 1 && !h->validate && h->small_miss != small_key;
  if (!small_try) {
    CK(cudaMemsetAsync(c_rpt, 0, sizeof(int64_t), h->stream));
    CK(cudaMemsetAsync(h->acc.p, 0, sizeof(DevAcc), h->stream));
  }
  if (m == 0) {
    CK(cudaStreamSynchronize(h->stream));
    h->nnzc = 0; h->nnza = 0; h->nnzb = 0;
    *c_nnz = 0;
    if (nprod_out) *nprod_out = 0;
    h->state = 1;
    CK(leave(h));
    return SPGEMM_OK;
  }
  ALLOC(h->nprod, sizeof(int64_t) * m);
  ALLOC(h->grp1, m);
  ALLOC(h->grp2, m);
  ALLOC(h->perm1, sizeof(int32_t) * m);
  ALLOC(h->perm2, sizeof(int32_t) * m);
  ALLOC(h->tiles, scan_workspace_bytes(m));
  if (h->range_hash) {
    ALLOC(h->bmm, sizeof(int2) * std::max<int64_t>(k, 1));
    ALLOC(h->binfo, sizeof(int4) * std::max<int64_t>(k, 1));  // {lo, hi, length} of every B row (step 1)
    ALLOC(h->rlohi, sizeof(int2) * m);
    ALLOC(h->defer_b, sizeof(int32_t) * std::max<int64_t>(k, 1));
  }
  if (h->timing) CK(cudaEventRecord(h->ev[0], h->stream));
  if (h->validate) {
    // checked before any kernel indexes B through col_A or walks rpt (an out-of-range column
    // would otherwise fault in the n_prod pass instead of returning SPGEMM_ERR_INVALID_INPUT)
    CK(launch_validate(h->stream, m, k, n, a_rpt, a_col, b_rpt, b_col, &dacc->err_flags));
    ++launches;
    CK(cudaMemcpyAsync(&h->hacc->err_flags, &dacc->err_flags, sizeof(int), cudaMemcpyDeviceToHost, h->stream));
    CK(cudaStreamSynchronize(h->stream));
    if (h->hacc->err_flags & 1)
      return fail(h, SPGEMM_ERR_INVALID_INPUT, "input validation failed (rpt not monotone or col out of range)");
  }
  // Small matrices: thread-per-row symbolic count with n_prod (Alg. 2) in the same pass and a
  // register table (rows with n_prod_i <= kSmallCap), then the rpt scan and one sync; rows above
  // the cap send the call down the general grouped path below.
  h->small = false;
  if (small_try) {
    // zero the counters, count, scan, copy the counters back: one captured segment (one graph
    // launch per call once the pointers repeat)
    const std::vector<long long> topo = {3, m, k, n, (long long)group_events(h)};
    const std::vector<long long> ptrs = {(long long)a_rpt, (long long)a_col, (long long)b_rpt, (long long)b_col,
                                         (long long)c_rpt, (long long)h->acc.p, (long long)h->nprod.p,
                                         (long long)h->hacc};
    auto enqueue = [&]() -> spgemm_status_t {
      CK(cudaMemsetAsync(c_rpt, 0, sizeof(int64_t), h->stream));
      CK(cudaMemsetAsync(h->acc.p, 0, sizeof(DevAcc), h->stream));
      CK(launch_small_symbolic(h->stream, m, k, a_rpt, a_col, b_rpt, b_col, c_rpt + 1,
                               static_cast<int64_t*>(h->nprod.p), dacc));
      // the scan kernel writes the counters straight to the pinned host copy (one graph node less)
      CK(launch_scan_small(h->stream, m, c_rpt, dacc, h->hacc_dev));
      return SPGEMM_OK;
    };
    const spgemm_status_t ss = run_graph(h, h->gsmall, topo, ptrs, enqueue);
    if (ss != SPGEMM_OK) return ss;
    const int nl = 2;
    CK(cudaStreamSynchronize(h->stream));  // the only host sync of the small path: nnz(C)
    if (h->hacc->small_overflow == 0) {
      h->snap1 = h->snap2 = *h->hacc;
      h->small = true;
      h->nnza = h->hacc->ends[1] - h->hacc->ends[0];
      h->nnzb = h->hacc->ends[3] - h->hacc->ends[2];
      h->nnzc = h->snap2.nnzc;
      *c_nnz = h->nnzc;
      if (nprod_out) *nprod_out = (int64_t)h->snap1.total_nprod;
      if (h->timing) {
        CK(cudaEventRecord(h->ev[3], h->stream));
        h->gtimed_phases = false;
      }
      spgemm_stats_t& st = h->stats;
      st.nnz_a = h->nnza; st.nnz_b = h->nnzb; st.nnz_c = h->nnzc;
      st.nprod = (int64_t)h->snap1.total_nprod;
      st.max_row_nprod = (int64_t)h->snap1.max_nprod;
      st.sym_rows[0] = st.num_rows[0] = m;
      st.sym_nprod[0] = st.num_nprod[0] = st.nprod;
      st.sym_nnza[0] = st.num_nnza[0] = h->nnza;
      st.num_nnzc[0] = h->nnzc;
      h->gkind[0][0] = SPGEMM_KERNEL_TINY;
      h->group_sums_done = true;
      st.kernel_launches_symbolic = launches + 1 + nl;
      h->state = 1;
      CK(leave(h));
      return SPGEMM_OK;
    }
    h->small_miss = small_key;  // the same inputs go straight to the grouped path next time
    CK(cudaMemsetAsync(c_rpt, 0, sizeof(int64_t), h->stream));  // general path from scratch
    CK(cudaMemsetAsync(h->acc.p, 0, sizeof(DevAcc), h->stream));
  }
  // (1)+(2): n_prod per row (Alg. 2), column spans, group ids / histogram
  {
    int nl = 0;
    CK(launch_nprod_group(h->stream, m, k, a_rpt, a_col, b_rpt, b_col, static_cast<int2*>(h->bmm.p),
                          static_cast<int4*>(h->binfo.p),
                          static_cast<int64_t*>(h->nprod.p), static_cast<int2*>(h->rlohi.p),
                          static_cast<uint8_t*>(h->grp1.p), c_rpt, dacc, sym_bounds(h),
                          static_cast<int32_t*>(h->perm1.p), static_cast<int32_t*>(h->defer_b.p), &nl));
    launches += nl;
  }
  CK(cudaMemcpyAsync(h->hacc, dacc, sizeof(DevAcc), cudaMemcpyDeviceToHost, h->stream));
  CK(cudaMemcpyAsync(h->hends + 0, a_rpt, sizeof(long long), cudaMemcpyDeviceToHost, h->stream));
  CK(cudaMemcpyAsync(h->hends + 1, a_rpt + m, sizeof(long long), cudaMemcpyDeviceToHost, h->stream));
  CK(cudaMemcpyAsync(h->hends + 2, b_rpt, sizeof(long long), cudaMemcpyDeviceToHost, h->stream));
  CK(cudaMemcpyAsync(h->hends + 3, b_rpt + k, sizeof(long long), cudaMemcpyDeviceToHost, h->stream));
  CK(cudaStreamSynchronize(h->stream));  // sync 1: group sizes
  h->snap1 = *h->hacc;
  if (h->snap1.err_flags & 1) return fail(h, SPGEMM_ERR_INVALID_INPUT, "input validation failed (rpt not monotone or col out of range)");
  h->nnza = h->hends[1] - h->hends[0];
  h->nnzb = h->hends[3] - h->hends[2];
  h->vw_log2 = auto_vw_log2(h);

  const Offsets off1 = offsets_of(h->snap1.sym_rows, kNumSymGroups);
  // (3) symbolic hash counting per group
  // optimistic-group rows counted exactly by the chunked rank-count kernel need no overflow lists
  // or global slabs (rank_cnt_on(kSymOptimistic) below).  Only with >= 4 rows per SM: one CTA per
  // row walks its products twice, so a handful of rows leaves the GPU idle behind the largest
  // (measured: R-MAT s22, 1811 rows, 1.95 -> 0.65 ms; s20, 211 rows, 0.04 -> 0.10 ms)
  const bool opt_exact = h->rank_acc && h->rank_big_sym && h->rlohi.p != nullptr && h->sym_min_group < 0 &&
                         (h->rank_big_sym == 2 || (long long)h->snap1.sym_rows[kSymOptimistic] >= 4LL * h->num_sms) &&
                         rankcnt_smem_bytes(kSymOptimistic, (int)((n + 1023) / 1024 + 1)) <= kSmemLimit;
  const long long n_opt = opt_exact ? 0 : (long long)h->snap1.sym_rows[kSymOptimistic];
  const long long n_glob = (long long)h->snap1.sym_rows[kSymGlobal];
  if (n_opt > 0) {
    ALLOC(h->overflow, sizeof(int32_t) * n_opt);
    ALLOC(h->overflow2, sizeof(int32_t) * n_opt);
  }
  int glob_grid = 0;
  long long slab_T = 0;
  if (n_opt + n_glob > 0) {  // global tables: forced-global rows and rows beyond the cluster table
    const long long cap = std::min<long long>((long long)h->snap1.max_nprod, n);
    slab_T = std::max<long long>(64, next_pow2(2 * std::max<long long>(cap, 1)));
    const long long per = slab_T * 4;
    const long long by_budget = std::max<long long>(1, h->ws_budget / per);
    const long long want = n_glob + (h->use_cluster ? std::min<long long>(n_opt, 32) : n_opt);
    glob_grid = (int)std::min<long long>({want, 2LL * h->num_sms, by_budget});
    ALLOC(h->slab_sym, (size_t)(glob_grid * per));
  }
  SymArgs sa{};
  sa.a_rpt = a_rpt; sa.a_col = a_col; sa.b_rpt = b_rpt; sa.b_col = b_col;
  sa.c_cnt = c_rpt + 1;
  sa.vw_log2 = h->vw_log2;
  sa.long_len = long_len_of(h);
  sa.flat = flat_of(h) ? 1 : 0;
  sa.rlohi = static_cast<const int2*>(h->rlohi.p);
  sa.overflow_rows = static_cast<int32_t*>(h->overflow.p);
  sa.overflow_count = &dacc->overflow_count;
  const int T_opt = kSymGroups[kSymOptimistic].T, BS_opt = kSymGroups[kSymOptimistic].BS;
  // default fill limit 3/4 of the table: a linear-probe miss at load 3/4 costs ~8 probes, far less
  // than the cluster retry of a row that aborts (R-MAT s22: 1803 of 1815 optimistic rows aborted
  // at T/2, 333 at 3T/4; optimistic group 4.6 -> 0.5 ms)
  int lim = h->fill_limit > 0 ? h->fill_limit : T_opt * 3 / 4;
  sa.fill_limit = std::max(1, std::min(lim, T_opt - BS_opt - 1));
  sa.slab = static_cast<int*>(h->slab_sym.p);
  sa.slab_T = slab_T;
  sa.nprod = static_cast<int64_t*>(h->nprod.p);
  sa.n = n;
  sa.l1_words = (int)((n + 1023) / 1024 + 1);
  sa.err_flags = &dacc->err_flags;
  // batched paper-hash symbolic kernels for groups 2-9 (kernels_esc.cu)
  auto batch_sym_on = [&](int g) { return (h->batch & 1) && h->sym_min_group < 0 && g >= 2 && g <= 9; };
  auto wsort_sym_on = [&](int g) { return (h->wsort & 1) && h->sym_min_group < 0 && g >= 2 && g <= wsort_max_group(); };
  // rank-count kernels for the CTA-per-row groups (kernels_rankacc.cu; needs the column spans)
  auto rank_cnt_on = [&](int g) {
    if (g == kSymOptimistic) return opt_exact;  // level 1 costs W words against > 16384 products
    return h->rank_acc && h->rlohi.p != nullptr && h->sym_min_group < 0 && g >= 5 && g <= 9 &&
           rankcnt_smem_bytes(g, sa.l1_words) <= kSmemLimit &&
           (h->rank_l1_pct_sym == 0 || 100LL * sa.l1_words <= h->rank_l1_pct_sym * kSymGroups[g].upper);
  };
  // range rows: pattern bitmap (symbolic -> numeric gather), rwcap words per row of the group
  const long long n_range = (long long)h->snap1.sym_rows[kSymRange];
  h->range_num = false;
  int range_bw = 0;  // > 0: symbolic range rows by B-row bitmap union (words per B-row bitmap)
  if (n_range > 0) {
    if (h->range_warp == 1 && h->snap1.range_rmax <= 1024) {
      const int bw = range_wcap(h->snap1.range_rmax);
      const long long bytes = k * (long long)bw * 4;
      if (bytes <= h->ws_budget / 2) {
        ALLOC(h->bbits, (size_t)bytes);
        range_bw = bw;
      }
    }
    sa.rwcap = range_wcap(h->snap1.range_rmax);
    const long long bytes = n_range * sa.rwcap * 4;  // <= 256 B per range row
    if (bytes <= h->ws_budget) {
      ALLOC(h->rbits, (size_t)bytes);
      sa.rbits = static_cast<unsigned*>(h->rbits.p);
      h->range_num = h->snap1.b_unsorted == 0 && h->num_min_group < 0;
    }
  }
  const int32_t* perm1 = static_cast<const int32_t*>(h->perm1.p);
  // segment 2 of phase 1 (scatter, per-group kernels on forked streams, scan): captured once per
  // (inputs, workspace, group histogram, options) and replayed
  std::vector<long long> topo = {1, m, k, n, glob_grid, slab_T, h->vw_log2, sa.long_len, sa.flat, sa.fill_limit,
                                 h->use_cluster, h->cluster_fill, h->use_streams, h->timing, h->num_min_group,
                                 h->range_hash, (long long)group_events(h), h->range_warp, h->range_min_np,
                                 h->snap1.range_rmax, h->snap1.b_unsorted, (long long)h->range_num, range_bw,
                                 (long long)h->rank_acc, (long long)h->tiny, h->rank_l1_pct_sym,
                                 (long long)h->sym_min_group, (long long)h->batch, h->esc_pct, h->esc_mask,
                                 (long long)h->small_opt, (long long)h->wsort, (long long)h->rank_big_sym};
  for (int g = 0; g < kMaxGroups; ++g) topo.push_back((long long)h->snap1.sym_rows[g]);
  const std::vector<long long> ptrs = {(long long)a_rpt, (long long)a_col, (long long)b_rpt, (long long)b_col,
                                       (long long)c_rpt, (long long)h->perm1.p, (long long)h->acc.p,
                                       (long long)h->slab_sym.p, (long long)h->overflow.p, (long long)h->overflow2.p,
                                       (long long)h->grp2.p, (long long)h->rlohi.p, (long long)h->nprod.p,
                                       (long long)h->tiles.p, (long long)h->grp1.p, (long long)h->rbits.p,
                                       (long long)h->bbits.p, (long long)h->bmm.p};
  int seg_launches = 0;
  const bool ge = group_events(h);
  h->gtimed_phases = ge && h->timing;
  auto enqueue = [&]() -> spgemm_status_t {
    int launches = 0;
    CK(launch_group_scatter(h->stream, m, static_cast<uint8_t*>(h->grp1.p), off1, dacc->cursor[0],
                            static_cast<int32_t*>(h->perm1.p)));
    ++launches;
    if (ge) CK(cudaEventRecord(h->ev[1], h->stream));
    h->phase_streams = phase_concurrent(h, h->snap1.sym_rows, kNumSymGroups);
    CK(fork(h));
    for (int g = 0; g <= kSymOptimistic; ++g) {
      const long long rows = (long long)h->snap1.sym_rows[g];
      if (rows == 0) continue;
      cudaStream_t s = group_stream(h, g);
      if (ge) CK(cudaEventRecord(h->gstart[0][g], s));
      SymArgs ga = sa;
      ga.rows = perm1 + off1.off[g];
      ga.nrows = rows;
      const bool tiny_g = h->tiny >= 2 && h->sym_min_group < 0 && g <= 1;  // measured slower than the hash
      if (tiny_g) CK(launch_symbolic_tiny(s, g, ga));
      else if (wsort_sym_on(g)) CK(launch_symbolic_wsort(s, g, ga));
      else if (batch_sym_on(g)) CK(launch_symbolic_batch(s, g, ga));
      else if (rank_cnt_on(g)) CK(launch_symbolic_rankcnt(s, g, ga));
      else CK(launch_symbolic_group(s, g, ga, h->num_sms));
      h->gkind[0][g] = tiny_g ? SPGEMM_KERNEL_TINY : wsort_sym_on(g) ? SPGEMM_KERNEL_WSORT : batch_sym_on(g) ? SPGEMM_KERNEL_BATCH
                     : rank_cnt_on(g) ? SPGEMM_KERNEL_RANK : SPGEMM_KERNEL_HASH;
      ++launches;
      if (g == kSymOptimistic && !opt_exact) {  // PAPER.md:155 "After this first phase ... global memory"
        SymArgs gb = sa;
        gb.rows = perm1 + off1.off[kSymGlobal];
        gb.nrows = n_glob;
        if (h->use_cluster) {  // overflow rows -> cluster DSMEM table -> (overflow2) global table
          SymArgs cb = sa;
          cb.nrows = 0;
          const int climit = h->cluster_fill > 0 ? std::min(h->cluster_fill, cluster_capacity_sym() / 2)
                                                 : cluster_capacity_sym() / 2;
          CK(launch_symbolic_cluster(s, cb, nullptr, &dacc->overflow_count, static_cast<int32_t*>(h->overflow2.p),
                                     &dacc->overflow2_count, climit, (int)n_opt));
          ++launches;
          gb.overflow2_rows = static_cast<const int32_t*>(h->overflow2.p);
          gb.dev_count2 = &dacc->overflow2_count;
        } else {
          gb.overflow2_rows = static_cast<const int32_t*>(h->overflow.p);
          gb.dev_count2 = &dacc->overflow_count;
        }
        CK(launch_symbolic_global(s, gb, glob_grid));
        ++launches;
        if (glob_grid > 0) h->gkind[0][kSymGlobal] = SPGEMM_KERNEL_GLOBAL;
      }
      if (ge) CK(cudaEventRecord(h->gstop[0][g], s));
      h->gtimed[0][g] = ge;
    }
    if (h->snap1.sym_rows[kSymRange] > 0) {  // range rows: warp-per-row offset tables
      cudaStream_t s = group_stream(h, kSymRange);
      if (ge) CK(cudaEventRecord(h->gstart[0][kSymRange], s));
      SymArgs ra = sa;
      ra.rows = perm1 + off1.off[kSymRange];
      ra.nrows = (long long)h->snap1.sym_rows[kSymRange];
      if (range_bw > 0) {  // B-row bitmaps, then the bitmap-union count
        CK(launch_brow_bits(s, k, b_rpt, b_col, static_cast<const int2*>(h->bmm.p), static_cast<unsigned*>(h->bbits.p),
                            range_bw, &dacc->bbits_wmax, h->num_sms));
        CK(launch_symbolic_range_bits(s, ra, static_cast<const unsigned*>(h->bbits.p), range_bw,
                                      static_cast<const int2*>(h->bmm.p), &dacc->bbits_wmax, h->num_sms));
        launches += 2;
      } else {
        CK(launch_symbolic_range(s, ra, h->snap1.range_rmax, h->num_sms));
        ++launches;
      }
      if (ge) CK(cudaEventRecord(h->gstop[0][kSymRange], s));
      h->gtimed[0][kSymRange] = ge;
      h->gkind[0][kSymRange] = SPGEMM_KERNEL_RANGE;
    }
    if (n_opt == 0 && n_glob > 0) {  // forced global group only
      cudaStream_t s = group_stream(h, kSymGlobal);
      if (ge) CK(cudaEventRecord(h->gstart[0][kSymGlobal], s));
      SymArgs gb = sa;
      gb.rows = perm1 + off1.off[kSymGlobal];
      gb.nrows = n_glob;
      gb.dev_count2 = nullptr;
      CK(launch_symbolic_global(s, gb, glob_grid));
      ++launches;
      if (ge) CK(cudaEventRecord(h->gstop[0][kSymGlobal], s));
      h->gtimed[0][kSymGlobal] = ge;
      h->gkind[0][kSymGlobal] = SPGEMM_KERNEL_GLOBAL;
    }
    CK(join(h));
    if (ge) CK(cudaEventRecord(h->ev[2], h->stream));

    // (4) rpt_C = prefix sum, fused with (6) grouping by nnz_i
    int nl = 0;
    // batched numeric rows need the column spans (bucket ranges) and no forced numeric group
    const bool esc_on = (h->batch & 2) && h->rlohi.p != nullptr && h->num_min_group < 0;
    const EscSel esc{esc_on ? static_cast<const int64_t*>(h->nprod.p) : nullptr, (int)std::min<long long>(h->esc_pct, 1 << 30),
                     (unsigned)(h->esc_mask < 0 ? esc_auto_mask(h) : h->esc_mask)};
    CK(launch_scan_and_group(h->stream, m, c_rpt, static_cast<const uint8_t*>(h->grp1.p),
                             static_cast<uint8_t*>(h->grp2.p), dacc, num_bounds(h), esc,
                             static_cast<long long*>(h->tiles.p), &nl));
    launches += nl;
    
    seg_launches = launches;
    return SPGEMM_OK;
  };
  {
    seg_launches = -1;
    const spgemm_status_t s2 = run_graph(h, h->gsym, topo, ptrs, enqueue);
    if (s2 != SPGEMM_OK) return s2;
    if (h->timing) CK(cudaEventRecord(h->ev[3], h->stream));
    if (seg_launches < 0) {  // replayed without enqueueing
      seg_launches = h->gsym.launches;
      memcpy(h->gtimed[0], h->gsym.timed, sizeof h->gsym.timed);
      memcpy(h->gkind[0], h->gsym.kind, sizeof h->gsym.kind);
    } else {
      h->gsym.launches = seg_launches;
      memcpy(h->gsym.timed, h->gtimed[0], sizeof h->gsym.timed);
      memcpy(h->gsym.kind, h->gkind[0], sizeof h->gsym.kind);
    }
  }
  launches += seg_launches;
  CK(cudaMemcpyAsync(h->hacc, dacc, sizeof(DevAcc), cudaMemcpyDeviceToHost, h->stream));
  CK(cudaStreamSynchronize(h->stream));  // sync 2: nnz(C) to the host
  h->snap2 = *h->hacc;
  h->nnzc = h->snap2.nnzc;
  *c_nnz = h->nnzc;
  if (nprod_out) *nprod_out = (int64_t)h->snap1.total_nprod;

  spgemm_stats_t& st = h->stats;
  st.nnz_a = h->nnza; st.nnz_b = h->nnzb; st.nnz_c = h->nnzc;
  st.nprod = (int64_t)h->snap1.total_nprod;
  st.max_row_nprod = (int64_t)h->snap1.max_nprod;
  st.max_row_nnz = (int64_t)h->snap2.max_nnz;
  for (int g = 0; g < kMaxGroups; ++g) {
    st.sym_rows[g] = (int64_t)h->snap1.sym_rows[g];
    st.num_rows[g] = (int64_t)h->snap2.num_rows[g];
  }
  h->group_sums_done = false;
  st.sym_overflow_rows = h->snap2.overflow_count;
  st.sym_overflow2_rows = h->snap2.overflow2_count;
  st.kernel_launches_symbolic = launches;
  h->state = 1;
  CK(leave(h));
  return SPGEMM_OK;
}

static spgemm_status_t ensure_perm2(spgemm_handle_t h) {
  if (h->perm2_ready || h->m == 0) return SPGEMM_OK;
  const Offsets off2 = offsets_of(h->snap2.num_rows, kNumNumGroups);
  DevAcc* dacc = static_cast<DevAcc*>(h->acc.p);
  CK(launch_group_scatter(h->stream, h->m, static_cast<uint8_t*>(h->grp2.p), off2, dacc->cursor[1],
                          static_cast<int32_t*>(h->perm2.p)));
  h->stats.kernel_launches_numeric += 1;
  h->perm2_ready = true;
  return SPGEMM_OK;
}

spgemm_status_t spgemm_numeric(spgemm_handle_t h, spgemm_dtype_t dt, const void* a_val, const void* b_val,
                               int32_t* c_col, void* c_val) {
  if (!h) return SPGEMM_ERR_INVALID_ARG;
  if (h->state != 1) return fail(h, SPGEMM_ERR_BAD_STATE, "spgemm_numeric before spgemm_symbolic");
  if (dt != SPGEMM_F32 && dt != SPGEMM_F64) return fail(h, SPGEMM_ERR_INVALID_ARG, "bad dtype");
  if (h->nnzc > 0 && (!c_col || !c_val)) return fail(h, SPGEMM_ERR_INVALID_ARG, "NULL output pointer");
  if (h->nnza > 0 && !a_val) return fail(h, SPGEMM_ERR_INVALID_ARG, "NULL a_val");
  if (h->nnzb > 0 && !b_val) return fail(h, SPGEMM_ERR_INVALID_ARG, "NULL b_val");
  DeviceGuard dg(h->device);
  CK(enter(h));
  h->stats.kernel_launches_numeric = 0;
  memset(h->gtimed[1], 0, sizeof h->gtimed[1]);
  memset(h->gkind[1], 0, sizeof h->gkind[1]);
  h->numeric_done = true;
  if (h->timing) CK(cudaEventRecord(h->ev[4], h->stream));
  if (h->small && h->nnzc > 0) {  // small-matrix path: one thread-per-row launch (kernels_tiny.cu)
    NumArgs na{};
    na.a_rpt = h->a_rpt; na.a_col = h->a_col; na.a_val = a_val;
    na.b_rpt = h->b_rpt; na.b_col = h->b_col; na.b_val = b_val;
    na.c_rpt = h->c_rpt; na.c_col = c_col; na.c_val = c_val;
    na.err_flags = &static_cast<DevAcc*>(h->acc.p)->err_flags;
    CK(launch_small_numeric(h->stream, dt == SPGEMM_F64, na, h->m));
    h->gkind[1][0] = SPGEMM_KERNEL_TINY;
    h->stats.kernel_launches_numeric = 1;
  } else if (h->m > 0 && h->nnzc > 0) {
    spgemm_status_t s = ensure_perm2(h);
    if (s != SPGEMM_OK) return s;
    const bool fp64 = dt == SPGEMM_F64;
    const long long vs = fp64 ? 8 : 4;
    const Offsets off2 = offsets_of(h->snap2.num_rows, kNumNumGroups);
    const Offsets off1 = offsets_of(h->snap1.sym_rows, kNumSymGroups);
    DevAcc* dacc = static_cast<DevAcc*>(h->acc.p);
    NumArgs na{};
    na.a_rpt = h->a_rpt; na.a_col = h->a_col; na.a_val = a_val;
    na.b_rpt = h->b_rpt; na.b_col = h->b_col; na.b_val = b_val;
    na.c_rpt = h->c_rpt; na.c_col = c_col; na.c_val = c_val;
    na.vw_log2 = h->vw_log2;
    na.long_len = long_len_of(h);
    na.flat = flat_of(h) ? 1 : 0;
    na.rlohi = static_cast<const int2*>(h->rlohi.p);
    na.priv_ok = h->snap1.b_unsorted ? 0 : 1;
    na.err_flags = &dacc->err_flags;
    na.l1_words = h->bitmap_rank ? (int)((h->n + 1023) / 1024 + 1) : 0;
    na.nprod = static_cast<const int64_t*>(h->nprod.p);
    // rank-indexed accumulation for the CTA-per-row groups (needs the column spans; the forced
    // paths keep the paper hash)
    const int l1w_rank = (int)((h->n + 1023) / 1024 + 1);
    // The CTA-group rank kernels hold <= KP*TPR (>= 2x the group's nnz bound) products per row in
    // registers; rows beyond that re-walk their products three times, which loses to the paper
    // hash when rows compress well (QCD-like: n_prod/nnz = 7.2).  Decided per call from the
    // global compression n_prod / nnz(C) (known at sync 2).
    const bool low_compression = (double)h->snap1.total_nprod <= 2.5 * (double)h->nnzc;
    auto rank_acc_on = [&](int g) {
      return h->rank_acc && low_compression && h->rlohi.p != nullptr && h->num_min_group < 0 && g >= 3 && g <= 9 &&
             rankacc_smem_bytes(g, fp64, l1w_rank) <= kSmemLimit &&
             (h->rank_l1_pct == 0 || 100LL * l1w_rank <= h->rank_l1_pct * kNumGroups[g].upper);
    };
    // cluster groups (clusters of 2/4/8 CTAs): bitmap + prefix scratch per resident cluster
    const long long cwords = h->n / 32 + 2;
    const long long cstride = (2 * cwords * 4 + 255) & ~255LL;
    long long ccount[3] = {0, 0, 0}, ctotal = 0;
    // rows above the CTA groups: rank-indexed accumulation with one CTA per row (level-2 bitmap
    // and prefix in a per-CTA global slab of 8 B per output entry), else the DSMEM cluster tables
    const bool big_rank = h->rank_acc && h->rlohi.p != nullptr && h->num_min_group < 0 &&
                          rankbig_smem_bytes(fp64, l1w_rank) <= kSmemLimit;
    long long bstride[3] = {0, 0, 0}, bgrid[3] = {0, 0, 0}, btotal = 0;
    // numeric group 9 on the persistent shared-memory rank kernel (RANK_MID)
    const bool mid_rank = h->rank_mid == 1 && h->snap2.num_rows[kNumCluster - 1] > 0 && rank_acc_on(kNumCluster - 1) &&
                          kNumGroups[kNumCluster - 1].upper <= kRankMidSharedL2 &&
                          rankbig_smem_bytes(fp64, l1w_rank, 2) <= kSmemLimit / 2;
    // big groups c < rank_big_max take the rank-big kernel, the others the DSMEM cluster tables
    auto big_rank_c = [&](int c) { return big_rank && c < h->rank_big_max; };
    for (int c = 0; c < 3; ++c) {
      const long long rows_c = (long long)h->snap2.num_rows[kNumCluster + c];
      if (rows_c == 0) continue;
      if (big_rank_c(c)) {
        bstride[c] = (kNumGroups[kNumCluster + c].upper * 8 + 16 + 255) & ~255LL;
        bgrid[c] = std::min<long long>(rows_c, h->num_sms);
        btotal += bgrid[c] * bstride[c];
        continue;
      }
      int nc = 0;
      CK(launch_numeric_cluster(h->stream, fp64, 2 << c, na, &nc));
      ccount[c] = std::min<long long>(nc, rows_c);
      ctotal += ccount[c];
    }
    // one slab buffer: cluster regions first, rank-big regions after them
    if (ctotal > 0 || btotal > 0) ALLOC(h->num_slab_c, (size_t)(ctotal * cstride + btotal));
    const long long n_glob = (long long)h->snap2.num_rows[kNumGlobal];
    int glob_grid = 0;
    if (n_glob > 0) {
      const long long maxn = std::max<long long>(1, (long long)h->snap2.max_nnz);
      const long long T = std::max<long long>(64, next_pow2(2 * maxn));
      const long long words = h->n / 32 + 2;  // bitmap over any column range [lo, hi]
      const long long stride = ((T * vs + T * 4 + 2 * words * 4) + 255) & ~255LL;
      const long long by_budget = std::max<long long>(1, h->ws_budget / stride);
      glob_grid = (int)std::min<long long>({n_glob, 2LL * h->num_sms, by_budget});
      ALLOC(h->num_slab, (size_t)(glob_grid * stride));
      na.bitmap_words = words;
      na.slab = h->num_slab.p; na.slab_T = T; na.slab_stride = stride; na.max_nnz = maxn;
    }
    const int32_t* perm2 = static_cast<const int32_t*>(h->perm2.p);
    // phase 2 (per-group kernels on forked streams): captured once per key and replayed (e.g.
    // numeric re-runs with new values of the same structure, or repeated multiplies)
    std::vector<long long> topo = {2, (long long)fp64, glob_grid, ctotal, btotal, h->vw_log2, na.long_len, na.flat,
                                   na.priv_ok, h->use_streams, h->timing, h->m, h->n, h->nnzc, (long long)group_events(h),
                                   h->snap1.range_rmax, (long long)na.l1_words, (long long)h->rank_acc, (long long)h->tiny,
                                   (long long)low_compression, h->rank_l1_pct, (long long)h->bitmap_rank,
                                   (long long)h->num_min_group, (long long)big_rank, (long long)h->rank_big_shared, (long long)mid_rank, (long long)h->rank_mid, (long long)h->rank_gout, (long long)h->rank_big_max, (long long)h->snap2.max_nnz,
                                   na.slab_T, na.slab_stride, cstride, (long long)na.bitmap_words, (long long)h->wsort};
    for (int g = 0; g < kMaxGroups; ++g) topo.push_back((long long)h->snap2.num_rows[g]);
    const std::vector<long long> ptrs = {(long long)a_val, (long long)b_val, (long long)c_col, (long long)c_val,
                                         (long long)h->c_rpt, (long long)h->a_rpt, (long long)h->a_col,
                                         (long long)h->b_rpt, (long long)h->b_col, (long long)perm2, (long long)h->acc.p,
                                         (long long)h->rlohi.p, (long long)h->num_slab.p, (long long)h->num_slab_c.p,
                                         (long long)h->rbits.p, (long long)h->perm1.p};
    const bool ge = group_events(h);
    auto enqueue = [&]() -> spgemm_status_t {
      if (ctotal > 0 || btotal > 0 || mid_rank)
        CK(cudaMemsetAsync(dacc->row_counter, 0, sizeof(dacc->row_counter), h->stream));
      h->phase_streams = phase_concurrent(h, h->snap2.num_rows, kNumNumGroups);
      CK(fork(h));
      for (int g = 0; g < kNumNumGroups; ++g) {
        const long long rows = (long long)h->snap2.num_rows[g];
        if (rows == 0) continue;
        cudaStream_t st = group_stream(h, g);
        if (ge) CK(cudaEventRecord(h->gstart[1][g], st));
        NumArgs ga = na;
        ga.rows = perm2 + off2.off[g];
        ga.nrows = rows;
        if (g >= kNumEscBase) {  // weakly compressing rows grouped by n_prod: warp-sorted or ESC batches
          const int sg = g - kNumEscBase + kEscSymLo;
          if ((h->wsort & 2) && sg <= wsort_max_group()) {
            h->gkind[1][g] = SPGEMM_KERNEL_WSORT;
            CK(launch_numeric_wsort(st, sg, fp64, ga));
          } else {
            h->gkind[1][g] = SPGEMM_KERNEL_ESC;
            CK(launch_numeric_esc(st, sg, fp64, ga));
          }
        } else if (g == kNumGlobal) {
          h->gkind[1][g] = SPGEMM_KERNEL_GLOBAL;
          CK(launch_numeric_global(st, fp64, ga, glob_grid));
        } else if (g == kNumRange) {
          // the symbolic range rows in their phase-1 order (the bitmap's row index)
          NumArgs ra = ga;
          ra.rows = static_cast<const int32_t*>(h->perm1.p) + off1.off[kSymRange];
          ra.nrows = (long long)h->snap1.sym_rows[kSymRange];
          ra.rbits = static_cast<const unsigned*>(h->rbits.p);
          ra.rwcap = range_wcap(h->snap1.range_rmax);
          h->gkind[1][g] = SPGEMM_KERNEL_RANGE;
          CK(launch_numeric_range(st, fp64, ra, h->snap1.range_rmax, h->num_sms));
        } else if (g >= kNumCluster && g < kNumCluster + 3) {
          const int c = g - kNumCluster;
          long long before = 0;
          for (int q = 0; q < c; ++q) before += ccount[q];
          NumArgs gc = ga;
          gc.slab = static_cast<unsigned char*>(h->num_slab_c.p) + before * cstride;
          gc.bitmap_words = cwords;
          gc.slab_stride = cstride;
          gc.row_counter = dacc->row_counter + c;
          const char* pg = getenv("SPGEMM_PROF_GROUP");  // diagnostics: per-row phase timestamps
          if (pg && atoi(pg) == g && !graphs_on(h)) {
            CK(cudaMalloc(&gc.prof, sizeof(unsigned long long) * 4 * rows));
            CK(cudaMemset(gc.prof, 0, sizeof(unsigned long long) * 4 * rows));
          }
          if (big_rank_c(c) && c == 0 && h->rank_big_shared == 2 && rankout_smem_bytes(g, fp64, l1w_rank) <= kSmemLimit) {
            // group 10: products in registers, output reduced into C, one 1024-thread CTA per row
            NumArgs ro = ga;
            ro.l1_words = l1w_rank;
            CK(launch_numeric_rankout(st, g, fp64, ro));
            h->gkind[1][g] = SPGEMM_KERNEL_RANK;
          } else if (big_rank_c(c)) {
            long long boff = ctotal * cstride;
            for (int q = 0; q < c; ++q) boff += bgrid[q] * bstride[q];
            gc.slab = static_cast<unsigned char*>(h->num_slab_c.p) + boff;
            gc.slab_stride = bstride[c];
            gc.slab_T = (long long)kNumGroups[kNumCluster + c].upper;
            gc.l1_words = l1w_rank;
            // group 10 (nnz_i <= 24576): level 2 in shared memory when it fits beside level 1
            const bool shl2 = c == 0 && h->rank_big_shared && kNumGroups[kNumCluster].upper <= kRankBigSharedL2 &&
                              rankbig_smem_bytes(fp64, l1w_rank, 1) <= kSmemLimit;
            CK(launch_numeric_rankbig(st, fp64, gc, (int)bgrid[c], shl2 ? 1 : 0));
            h->gkind[1][g] = SPGEMM_KERNEL_RANK_BIG;
          } else {
            CK(launch_numeric_cluster(st, fp64, 2 << c, gc, nullptr));
            h->gkind[1][g] = SPGEMM_KERNEL_CLUSTER;
          }
          if (gc.prof) {
            std::vector<unsigned long long> hp((size_t)(4 * rows));
            CK(cudaStreamSynchronize(st));
            CK(cudaMemcpy(hp.data(), gc.prof, hp.size() * 8, cudaMemcpyDeviceToHost));
            cudaFree(gc.prof);
            const char* out = getenv("SPGEMM_PROF_OUT");
            if (FILE* f = fopen(out ? out : "spgemm_prof.bin", "wb")) {
              fwrite(hp.data(), 8, hp.size(), f);
              fclose(f);
            }
          }
        } else {
          const char* pg = getenv("SPGEMM_PROF_GROUP");  // diagnostics: per-row phase timestamps
          if (pg && atoi(pg) == g && !graphs_on(h)) {
            CK(cudaMalloc(&ga.prof, sizeof(unsigned long long) * 4 * rows));
            CK(cudaMemset(ga.prof, 0, sizeof(unsigned long long) * 4 * rows));
          }
          if (h->tiny && h->num_min_group < 0 && g <= 1) {
            CK(launch_numeric_tiny(st, g, fp64, ga));
            h->gkind[1][g] = SPGEMM_KERNEL_TINY;
          } else if (rank_acc_on(g) && ((g == kNumCluster - 1 && h->rank_mid == 2) || (g < kNumCluster - 1 && h->rank_gout)) &&
                     rankout_smem_bytes(g, fp64, l1w_rank) <= (g == kNumCluster - 1 ? kSmemLimit / 2 : kSmemLimit)) {
            NumArgs ra = ga;
            ra.l1_words = l1w_rank;
            CK(launch_numeric_rankout(st, g, fp64, ra));
            h->gkind[1][g] = SPGEMM_KERNEL_RANK;
          } else if (rank_acc_on(g) && g == kNumCluster - 1 && mid_rank) {
            // group 9: persistent rank kernel, two 512-thread CTAs per SM, level 2 in shared
            // memory, values reduced into C
            NumArgs ra = ga;
            ra.l1_words = l1w_rank;
            ra.row_counter = dacc->row_counter + 3;
            CK(launch_numeric_rankbig(st, fp64, ra, (int)std::min<long long>(rows, 2LL * h->num_sms), 2));
            h->gkind[1][g] = SPGEMM_KERNEL_RANK_BIG;
          } else if (rank_acc_on(g)) {
            NumArgs ra = ga;
            ra.l1_words = l1w_rank;
            CK(launch_numeric_rankacc(st, g, fp64, ra));
            h->gkind[1][g] = SPGEMM_KERNEL_RANK;
          } else {
            NumArgs hb = ga;
            if (h->bitmap_rank == 1 && g < kNumNumBounds && (long long)hb.l1_words > kNumGroups[g].upper) hb.l1_words = 0;
            CK(launch_numeric_group(st, g, fp64, hb));
            h->gkind[1][g] = SPGEMM_KERNEL_HASH;
          }
          if (ga.prof) {
            std::vector<unsigned long long> hp((size_t)(4 * rows));
            CK(cudaStreamSynchronize(st));
            CK(cudaMemcpy(hp.data(), ga.prof, hp.size() * 8, cudaMemcpyDeviceToHost));
            cudaFree(ga.prof);
            const char* out = getenv("SPGEMM_PROF_OUT");
            if (FILE* f = fopen(out ? out : "spgemm_prof.bin", "wb")) {
              fwrite(hp.data(), 8, hp.size(), f);
              fclose(f);
            }
          }
        }
        h->stats.kernel_launches_numeric += 1;
        if (ge) CK(cudaEventRecord(h->gstop[1][g], st));
        h->gtimed[1][g] = ge;
      }
      CK(join(h));
      return SPGEMM_OK;
    };
    const long long before_launches = h->stats.kernel_launches_numeric;
    s = run_graph(h, h->gnum, topo, ptrs, enqueue);
    if (s != SPGEMM_OK) return s;
    if (h->stats.kernel_launches_numeric == before_launches) {  // replayed without enqueueing
      h->stats.kernel_launches_numeric += h->gnum.launches;
      memcpy(h->gtimed[1], h->gnum.timed, sizeof h->gnum.timed);
      memcpy(h->gkind[1], h->gnum.kind, sizeof h->gnum.kind);
    } else {
      h->gnum.launches = (int)(h->stats.kernel_launches_numeric - before_launches);
      memcpy(h->gnum.timed, h->gtimed[1], sizeof h->gnum.timed);
      memcpy(h->gnum.kind, h->gkind[1], sizeof h->gnum.kind);
    }
  }
  if (h->timing) CK(cudaEventRecord(h->ev[5], h->stream));
  CK(leave(h));
  return SPGEMM_OK;
}

spgemm_status_t spgemm_get_stats(spgemm_handle_t h, spgemm_stats_t* out) {
  if (!h || !out) return SPGEMM_ERR_INVALID_ARG;
  DeviceGuard dg(h->device);
  CK(enter(h));
  spgemm_stats_t st = h->stats;
  for (int g = 0; g < kMaxGroups; ++g) {
    st.sym_kernel[g] = h->gkind[0][g];
    st.num_kernel[g] = h->numeric_done ? h->gkind[1][g] : 0;
  }
  if (h->state == 1 && h->m > 0 && h->timing) {
    auto el = [&](cudaEvent_t a, cudaEvent_t b) -> float {
      float ms = 0.f;
      if (cudaEventSynchronize(b) != cudaSuccess || cudaEventElapsedTime(&ms, a, b) != cudaSuccess) {
        cudaGetLastError();
        return -1.f;
      }
      return ms;
    };
    if (h->gtimed_phases) {
      st.setup_ms = el(h->ev[0], h->ev[1]);
      st.symbolic_ms = el(h->ev[1], h->ev[2]);
      st.scan_ms = el(h->ev[2], h->ev[3]);
    } else {  // graph mode: phase 1 as a whole
      st.symbolic_ms = el(h->ev[0], h->ev[3]);
    }
    for (int g = 0; g < kMaxGroups; ++g) st.sym_group_ms[g] = h->gtimed[0][g] ? el(h->gstart[0][g], h->gstop[0][g]) : 0.f;
    if (h->numeric_done) {
      st.numeric_ms = el(h->ev[4], h->ev[5]);
      for (int g = 0; g < kMaxGroups; ++g) st.num_group_ms[g] = h->gtimed[1][g] ? el(h->gstart[1][g], h->gstop[1][g]) : 0.f;
      int flags = 0;
      if (cudaMemcpy(&flags, &static_cast<DevAcc*>(h->acc.p)->err_flags, sizeof(int), cudaMemcpyDeviceToHost) == cudaSuccess &&
          (flags & 2)) {
        *out = st;
        return fail(h, SPGEMM_ERR_INVALID_INPUT, "numeric row count disagreed with symbolic count");
      }
    }
  }
  if (h->state == 1 && h->m > 0) {
    if (!h->group_sums_done) {  // off the critical path: one extra kernel + copy, on demand
      DevAcc* dacc = static_cast<DevAcc*>(h->acc.p);
      CK(launch_group_stats(h->stream, h->m, static_cast<uint8_t*>(h->grp1.p), static_cast<uint8_t*>(h->grp2.p),
                            static_cast<int64_t*>(h->nprod.p), h->a_rpt, h->c_rpt, dacc));
      CK(cudaMemcpyAsync(h->hacc, dacc, sizeof(DevAcc), cudaMemcpyDeviceToHost, h->stream));
      CK(cudaStreamSynchronize(h->stream));
      for (int g = 0; g < kMaxGroups; ++g) {
        h->stats.sym_nprod[g] = (int64_t)h->hacc->sym_nprod[g];
        h->stats.sym_nnza[g] = (int64_t)h->hacc->sym_nnza[g];
        h->stats.num_nprod[g] = (int64_t)h->hacc->num_nprod[g];
        h->stats.num_nnza[g] = (int64_t)h->hacc->num_nnza[g];
        h->stats.num_nnzc[g] = (int64_t)h->hacc->num_nnzc[g];
      }
      h->group_sums_done = true;
    }
    for (int g = 0; g < kMaxGroups; ++g) {
      st.sym_nprod[g] = h->stats.sym_nprod[g];
      st.sym_nnza[g] = h->stats.sym_nnza[g];
      st.num_nprod[g] = h->stats.num_nprod[g];
      st.num_nnza[g] = h->stats.num_nnza[g];
      st.num_nnzc[g] = h->stats.num_nnzc[g];
    }
  }
  CK(leave(h));
  st.workspace_bytes = h->ws_cur;
  st.workspace_peak_bytes = h->ws_peak;
  *out = st;
  return SPGEMM_OK;
}

spgemm_status_t spgemm_get_grouping(spgemm_handle_t h, int phase, int64_t* nprod, int32_t* perm, int64_t* offsets) {
  if (!h || (phase != 1 && phase != 2)) return SPGEMM_ERR_INVALID_ARG;
  if (h->state != 1) return fail(h, SPGEMM_ERR_BAD_STATE, "no symbolic result");
  if (h->small)
    return fail(h, SPGEMM_ERR_BAD_STATE, "the small-matrix path builds no grouping (set SPGEMM_OPT_SMALL 0)");
  DeviceGuard dg(h->device);
  CK(enter(h));
  if (h->m == 0) {
    if (offsets) for (int g = 0; g <= (phase == 1 ? kNumSymGroups : kNumNumGroups); ++g) offsets[g] = 0;
    return SPGEMM_OK;
  }
  if (phase == 2) {
    spgemm_status_t s = ensure_perm2(h);
    if (s != SPGEMM_OK) return s;
  }
  CK(cudaStreamSynchronize(h->stream));
  if (nprod) CK(cudaMemcpy(nprod, h->nprod.p, sizeof(int64_t) * h->m, cudaMemcpyDeviceToHost));
  if (perm) CK(cudaMemcpy(perm, phase == 1 ? h->perm1.p : h->perm2.p, sizeof(int32_t) * h->m, cudaMemcpyDeviceToHost));
  if (offsets) {
    const int ng = phase == 1 ? kNumSymGroups : kNumNumGroups;
    const Offsets o = offsets_of(phase == 1 ? h->snap1.sym_rows : h->snap2.num_rows, ng);
    for (int g = 0; g <= ng; ++g) offsets[g] = o.off[g];
  }
  return SPGEMM_OK;
}

spgemm_status_t spgemm_row_partition(spgemm_handle_t h, int64_t m, int64_t k, const int64_t* a_rpt,
                                     const int32_t* a_col, const int64_t* b_rpt, int32_t nparts, int64_t* splits) {
  if (!h || !splits || !a_rpt || !b_rpt || m < 0 || k < 0 || nparts < 1) return SPGEMM_ERR_INVALID_ARG;
  if (!h->hacc) return fail(h, SPGEMM_ERR_BAD_STATE, "handle was not created successfully");
  DeviceGuard dg(h->device);
  CK(enter(h));
  Buf scan, tiles, dsplits;
  spgemm_status_t s = buf_alloc(h, scan, sizeof(int64_t) * (m + 1));
  if (s == SPGEMM_OK) s = buf_alloc(h, tiles, scan_workspace_bytes(m));
  if (s == SPGEMM_OK) s = buf_alloc(h, dsplits, sizeof(int64_t) * (nparts + 1));
  cudaError_t e = cudaSuccess;
  if (s == SPGEMM_OK) {
    int nl = 0;
    e = launch_partition(h->stream, m, a_rpt, a_col, b_rpt, static_cast<int64_t*>(scan.p),
                         static_cast<long long*>(tiles.p), nparts, static_cast<int64_t*>(dsplits.p), &nl);
    if (e == cudaSuccess)
      e = cudaMemcpyAsync(splits, dsplits.p, sizeof(int64_t) * (nparts + 1), cudaMemcpyDeviceToHost, h->stream);
    if (e == cudaSuccess) e = cudaStreamSynchronize(h->stream);
  }
  buf_free(h, scan);
  buf_free(h, tiles);
  buf_free(h, dsplits);
  if (s != SPGEMM_OK) return s;
  if (e != cudaSuccess) return fail_cuda(h, e, "spgemm_row_partition");
  CK(leave(h));
  return SPGEMM_OK;
}

}  // extern "C"
