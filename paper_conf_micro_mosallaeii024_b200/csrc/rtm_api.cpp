// rtm_api.cpp — C ABI of librtm (include/rtm.h): context, ingest, the window-reduce
// orchestration on one CUDA stream, result accessors and the multi-rank exchange.
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

#include <algorithm>
#include <vector>

#include "rtm.h"
#include "rtm_internal.h"

using namespace rtm;

namespace {

struct DevBuf {
  void *p = nullptr;
  size_t cap = 0;
};

struct Pinned {
  void *p = nullptr;
  size_t cap = 0;
};

struct Chunk {
  const void *ptr;
  uint64_t n;
};

constexpr uint32_t kGraphAutoMaxWindows = 64;  // RTM_GRAPHS_AUTO: calls of at most this many windows
constexpr size_t kGraphCacheSize = 8;           // launch shapes cached per context

enum KernelId { KT_SPLIT, KT_PARTITION, KT_EVENTS, KT_FOLD, KT_ORDER, KT_TOPK, KT_HANG, KT_PROGRESS, KT_MERGE,
                KT_SUBPART, KT_N };
const char *kKernelNames[KT_N] = {"k_prep", "k_partition", "k_events", "k_fold", "k_order_check",
                                  "k_topk", "k_hang", "k_progress", "k_merge", "k_subpart"};

}  // namespace

struct rtm_ctx {
  // registry
  uint32_t nb, nc, nk, nbins, ncw, k, H;
  int32_t bin_log = 8;
  int32_t rank_mode, device, rank, world, hang_mode;
  int64_t t0;
  rtm_allgather_fn allgather;
  void *allgather_user;
  cudaStream_t st;
  cudaStream_t st2 = nullptr;            // side stream (task events), joined per call
  cudaEvent_t ev_fork = nullptr, ev_join = nullptr;
  int n_sms;
  // CUDA graphs of the reduce launch sequence (rtm_use_graphs): one per launch shape, replayed with
  // the call's Params; valid while no workspace was reallocated (gen)
  struct GraphEntry {
    uint64_t key[3], gen, used;
    cudaGraph_t g;
    cudaGraphExec_t x;
    std::vector<cudaGraphNode_t> kn;      // kernel nodes
    std::vector<cudaKernelNodeParams> kp;  // their launch configurations
  };
  int32_t graph_mode = RTM_GRAPHS_AUTO;
  cudaStream_t cap_st = nullptr;  // capture stream (the context stream may be the legacy default stream)
  bool graph_broken = false;  // capture / instantiation unsupported here: direct launches only
  uint64_t gen = 0, graph_tick = 0;
  uint64_t graph_captures = 0, graph_replays = 0;  // rtm_graph_stats
  std::vector<GraphEntry> graphs;
  DevBuf cap, owner, elig, ktotal, rcp, elig_ids;
  DevBuf gid, bstat_g;      // rank-local numbering: global id per local buffer, table by global id
  DevBuf tkscr;             // per-slice top-k candidates (few-window calls)
  DevBuf mkey, rcp64;       // rank mode MEAN: per-(window, buffer) order keys, floor(2^64 / c)
  DevBuf tkey;              // rank mode MEAN, world > 1: the local top-k's order keys (exchange pack)
  DevBuf persist;           // windows-in-top-k counter per buffer (id space)
  DevBuf klive;             // progress bar ids in use
  std::vector<uint8_t> klive_h;
  std::vector<int64_t> ktotal0;  // bar totals registered at create (restored by reset)
  uint32_t cap_max = 0;          // largest registered capacity (the fold's 32-bit D condition)
  bool bars_dirty = true;        // registry changed since create / the last reset
  std::vector<uint32_t> link_off, link_dst;  // component connection graph (CSR by source)
  // value monitor: watched ids (as given), their local ids (~0: not on this rank), rings
  std::vector<uint32_t> gid_h;  // host copy of the global ids (rank-local numbering)
  std::vector<uint8_t> elig_h;  // host copy of elig (buffer owned by this rank)
  uint32_t n_watch = 0;
  uint32_t watch_ids[RTM_WATCH_MAX] = {0}, watch_local[RTM_WATCH_MAX] = {0};
  std::vector<rtm_watch_point> ring[RTM_WATCH_MAX];
  uint32_t ring_head[RTM_WATCH_MAX] = {0}, ring_n[RTM_WATCH_MAX] = {0};
  uint32_t n_global = 0, pack_nb = 0;
  uint32_t n_elig = 0;
  // persistent state
  DevBuf carry[2];
  int cur = 0;
  DevBuf run[2], kstart, kend, cstart, cend, flags;
  uint32_t epoch = 1;        // look-back flag value of the current / last call (never 0)
  bool merge_pending = false;  // rtm_window_reduce_local done, rtm_merge not yet
  bool tables_synced = true;   // world > 1: the last call's tables exchanged (rtm_tables_merge)
  bool ag_on_stream = false;   // the allgather callback is stream-ordered on `st` (no host sync)
  DevBuf gcum;                 // world > 1: merged cumulative START / END per bar [nk][2] i64
  DevBuf tpack, tgathered;     // on-demand tables exchange
  int64_t t_prev;
  int sticky = 0;
  // pending stream
  std::vector<Chunk> s_dev, e_dev;  // zero-copy device chunks
  DevBuf s_own, e_own;              // internal concatenation
  uint64_t s_own_n = 0, e_own_n = 0;
  // per-call workspaces
  DevBuf T, Bs, Be, rts, rte, treg_s, treg_e, tdesc, soff, stage, stage2, woff, smeta, emeta, lastlvl, res, kdelta, cdelta, active,
      anyfull, hung, unit_ctr, bstat, comps, pack, gathered, endkey, hsfx;
  Pinned h_small, h_res;
  // results of the last call
  bool have = false;
  uint32_t W = 0;
  std::vector<rtm_window_summary> sum;
  // results of the last call: views into the pinned host buffer h_res (valid until the next call)
  const unsigned long long *topk_h = nullptr;
  const uint32_t *topk_n_h = nullptr;
  const rtm_progress_entry *prog_h = nullptr;
  std::vector<int64_t> t_end_h;
  // profiling
  bool prof = false;
  KernelTimer timers[KT_N];
  std::vector<cudaEvent_t> ev_pool;
  struct Mark { int kid; cudaEvent_t a, b; uint64_t bytes; };
  std::vector<Mark> marks;
  size_t ev_next = 0;
};

namespace {

rtm_status cuda_fail(rtm_ctx *c, cudaError_t e, const char *what, int line) {
  static const bool dbg = getenv("RTM_DEBUG") != nullptr;
  if (dbg) fprintf(stderr, "[rtm] CUDA error %d (%s) at rtm_api.cpp:%d: %s\n", (int)e, cudaGetErrorString(e), line, what);
  cudaGetLastError();
  if (c) c->sticky = RTM_E_CUDA;
  return RTM_E_CUDA;
}

#define CK(call)                                                    \
  do {                                                              \
    cudaError_t e_ = (call);                                        \
    if (e_ != cudaSuccess) return cuda_fail(c, e_, #call, __LINE__); \
  } while (0)

rtm_status ensure(rtm_ctx *c, DevBuf &b, size_t bytes, bool zero_new = false) {
  if (bytes == 0) bytes = 8;
  if (b.cap >= bytes) return RTM_OK;
  if (b.p) cudaFree(b.p);
  b.p = nullptr;
  b.cap = 0;
  size_t want = bytes + bytes / 4;
  ++c->gen;  // cached CUDA graphs hold the old pointers
  cudaError_t e = cudaMalloc(&b.p, want);
  if (e != cudaSuccess) {
    cudaGetLastError();
    e = cudaMalloc(&b.p, bytes);
    want = bytes;
  }
  if (e != cudaSuccess) {
    cudaGetLastError();
    b.p = nullptr;
    c->sticky = RTM_E_NOMEM;
    return RTM_E_NOMEM;
  }
  b.cap = want;
  // stream-ordered: the kernels that first use the buffer run on the context stream
  if (zero_new && cudaMemsetAsync(b.p, 0, want, c->st) != cudaSuccess) return cuda_fail(c, cudaGetLastError(), "memset", __LINE__);
  return RTM_OK;
}

// grow keeping the first `keep` bytes (used for the ingest concatenation buffer)
rtm_status grow_keep(rtm_ctx *c, DevBuf &b, size_t bytes, size_t keep) {
  if (b.cap >= bytes) return RTM_OK;
  size_t want = std::max(bytes + bytes / 2, (size_t)1 << 20);
  void *np = nullptr;
  ++c->gen;
  if (cudaMalloc(&np, want) != cudaSuccess) {
    cudaGetLastError();
    c->sticky = RTM_E_NOMEM;
    return RTM_E_NOMEM;
  }
  if (keep) CK(cudaMemcpyAsync(np, b.p, keep, cudaMemcpyDeviceToDevice, c->st));
  CK(cudaStreamSynchronize(c->st));
  if (b.p) cudaFree(b.p);
  b.p = np;
  b.cap = want;
  return RTM_OK;
}

rtm_status ensure_pinned(rtm_ctx *c, Pinned &h, size_t bytes) {
  if (h.cap >= bytes) return RTM_OK;
  if (h.p) cudaFreeHost(h.p);
  h.p = nullptr;
  ++c->gen;
  size_t want = std::max(bytes + bytes / 4, (size_t)1 << 16);
  if (cudaMallocHost(&h.p, want) != cudaSuccess) {
    cudaGetLastError();
    h.cap = 0;
    c->sticky = RTM_E_NOMEM;
    return RTM_E_NOMEM;
  }
  h.cap = want;
  return RTM_OK;
}

void prof_begin(rtm_ctx *c, int kid, uint64_t bytes) {
  if (!c->prof) return;
  if (c->ev_next + 2 > c->ev_pool.size()) {
    for (int i = 0; i < 32; ++i) {
      cudaEvent_t e;
      cudaEventCreate(&e);
      c->ev_pool.push_back(e);
    }
  }
  rtm_ctx::Mark m;
  m.kid = kid;
  m.a = c->ev_pool[c->ev_next++];
  m.b = c->ev_pool[c->ev_next++];
  m.bytes = bytes;
  cudaEventRecord(m.a, c->st);
  c->marks.push_back(m);
}
void prof_end(rtm_ctx *c) {
  if (!c->prof || c->marks.empty()) return;
  cudaEventRecord(c->marks.back().b, c->st);
}
void prof_begin_on(rtm_ctx *c, int kid, uint64_t bytes, cudaStream_t st) {
  prof_begin(c, kid, bytes);  // records on c->st: re-record on the side stream
  if (c->prof && !c->marks.empty()) cudaEventRecord(c->marks.back().a, st);
}
void prof_end_on(rtm_ctx *c, cudaStream_t st) {
  if (!c->prof || c->marks.empty()) return;
  cudaEventRecord(c->marks.back().b, st);
}
void prof_collect(rtm_ctx *c) {  // after a stream sync
  for (auto &m : c->marks) {
    float ms = 0;
    if (cudaEventElapsedTime(&ms, m.a, m.b) == cudaSuccess) {
      c->timers[m.kid].launches++;
      c->timers[m.kid].total_ms += ms;
      c->timers[m.kid].algo_bytes += m.bytes;
    } else {
      cudaGetLastError();
    }
  }
  c->marks.clear();
  c->ev_next = 0;
}

#define LAUNCH(kid, bytes, stmt) \
  do {                           \
    prof_begin(c, kid, bytes);   \
    stmt;                        \
    prof_end(c);                 \
  } while (0)

void free_buf(DevBuf &b) {
  if (b.p) cudaFree(b.p);
  b.p = nullptr;
  b.cap = 0;
}

rtm_status zero_state(rtm_ctx *c) {
  ClearList cl;  // stream-ordered: the next call's kernels see the cleared state
  cl.add(c->carry[0].p, (size_t)c->nb * 2);
  cl.add(c->carry[1].p, (size_t)c->nb * 2);
  cl.add(c->run[0].p, (size_t)c->nc * 4);
  cl.add(c->run[1].p, (size_t)c->nc * 4);
  cl.add(c->kstart.p, (size_t)c->nk * 8);
  cl.add(c->kend.p, (size_t)c->nk * 8);
  cl.add(c->cstart.p, (size_t)c->nc * 8);
  cl.add(c->cend.p, (size_t)c->nc * 8);
  cl.add(c->persist.p, (size_t)(c->n_global ? c->n_global : c->nb) * 4);
  cl.add(c->gcum.p, (size_t)c->nk * 16);
  cl.add(c->cdelta.p, (size_t)c->nc * 16);
  launch_clear(cl, c->st);
  CK(cudaGetLastError());
  if (c->bars_dirty) {  // every registered bar live with its registered total (only after changes:
    c->klive_h.assign(c->nk, 1);  // reset sits inside streaming loops, keep it free of host syncs)
    CK(cudaMemcpyAsync(c->klive.p, c->klive_h.data(), c->nk, cudaMemcpyHostToDevice, c->st));
    CK(cudaMemcpyAsync(c->ktotal.p, c->ktotal0.data(), (size_t)c->nk * 8, cudaMemcpyHostToDevice, c->st));
    CK(cudaStreamSynchronize(c->st));  // pageable sources
    c->bars_dirty = false;
  }
  c->cur = 0;
  c->t_prev = c->t0;
  c->have = false;
  c->merge_pending = false;
  c->tables_synced = true;
  c->W = 0;
  c->s_dev.clear();
  c->e_dev.clear();
  c->s_own_n = c->e_own_n = 0;
  return RTM_OK;
}

// Pending stream of one kind as a single device array.
void pending(const std::vector<Chunk> &dev, const DevBuf &own, uint64_t own_n, const void **ptr, uint64_t *n) {
  if (own_n) { *ptr = own.p; *n = own_n; }
  else if (!dev.empty()) { *ptr = dev[0].ptr; *n = dev[0].n; }
  else { *ptr = nullptr; *n = 0; }
}

rtm_status append(rtm_ctx *c, std::vector<Chunk> &dev, DevBuf &own, uint64_t &own_n, const void *src, uint64_t n,
                  int32_t mem) {
  if (n == 0) return RTM_OK;
  const size_t rec = 16;
  if (mem == RTM_MEM_DEVICE && dev.empty() && own_n == 0) {
    dev.push_back({src, n});  // zero-copy
    return RTM_OK;
  }
  // move a pending zero-copy chunk into the internal buffer first
  if (!dev.empty()) {
    rtm_status s = grow_keep(c, own, (size_t)(own_n + dev[0].n) * rec, (size_t)own_n * rec);
    if (s) return s;
    CK(cudaMemcpyAsync((char *)own.p + own_n * rec, dev[0].ptr, dev[0].n * rec, cudaMemcpyDeviceToDevice, c->st));
    own_n += dev[0].n;
    dev.clear();
  }
  rtm_status s = grow_keep(c, own, (size_t)(own_n + n) * rec, (size_t)own_n * rec);
  if (s) return s;
  CK(cudaMemcpyAsync((char *)own.p + own_n * rec, src, n * rec,
                     mem == RTM_MEM_DEVICE ? cudaMemcpyDeviceToDevice : cudaMemcpyHostToDevice, c->st));
  own_n += n;
  return RTM_OK;
}

// The local (per-rank) part of a reduce call.  On success the device result arrays hold this
// rank's per-window results for n_windows windows.
// Per-call results, one device buffer and one pinned host buffer of the same layout (a single
// D2H copy per call): window fields | top-k | progress | top-k counts | status.
struct ResLayout {
  size_t win, topk, prog, topk_n, status, watch, bytes;
};
ResLayout res_layout(const rtm_ctx *c, uint32_t W) {
  ResLayout L;
  L.win = 0;
  L.topk = L.win + (size_t)kWinFields * W * 8;
  L.prog = L.topk + (size_t)W * c->k * 8;
  L.topk_n = L.prog + (size_t)W * c->nk * 5 * 8;
  L.status = L.topk_n + (((size_t)W * 4 + 15) & ~(size_t)15);
  L.watch = L.status + 16;  // value monitor points, only while buffers are watched
  L.bytes = L.watch + (c->n_watch ? (size_t)W * RTM_WATCH_MAX * sizeof(rtm_buffer_stat) : 0);
  return L;
}
void set_result_ptrs(rtm_ctx *c, uint32_t W, Params &p) {
  const ResLayout L = res_layout(c, W);
  char *d = (char *)c->res.p;
  p.win = (unsigned long long *)(d + L.win);
  p.topk = (unsigned long long *)(d + L.topk);
  p.prog = (long long *)(d + L.prog);
  p.topk_n = (uint32_t *)(d + L.topk_n);
  p.status = (uint32_t *)(d + L.status);
  p.n_watch = c->n_watch;
  for (uint32_t q = 0; q < RTM_WATCH_MAX; ++q) p.watch[q] = q < c->n_watch ? c->watch_local[q] : 0xFFFFFFFFu;
  p.wstat = (rtm_buffer_stat *)(d + L.watch);
}

// ---- CUDA graphs of the launch sequence (rtm_use_graphs) ------------------------------------
bool graph_use(const rtm_ctx *c, uint32_t W) {
#ifdef RTM_PHASE_TIMING
  (void)c; (void)W;
  return false;
#else
  if (c->prof || c->graph_broken) return false;
  return c->graph_mode == RTM_GRAPHS_ALWAYS || (c->graph_mode == RTM_GRAPHS_AUTO && W <= kGraphAutoMaxWindows);
#endif
}

void graph_free(rtm_ctx::GraphEntry &e) {
  if (e.x) cudaGraphExecDestroy(e.x);
  if (e.g) cudaGraphDestroy(e.g);
  e.x = nullptr;
  e.g = nullptr;
}

void graphs_clear(rtm_ctx *c) {
  for (auto &e : c->graphs) graph_free(e);
  c->graphs.clear();
}

// Replays the graph captured for this call's launch shape (capturing it first if needed).  A
// replay replaces every kernel node's arguments with this call's (Params; k_prep: Params, clear
// list, split buffers): the shape key fixes everything else - kernel variants, grids, shared
// memory, the memcpy of the window bounds from the pinned staging (its pointer is guarded by the
// workspace generation).
template <typename F>
rtm_status graph_launch(rtm_ctx *c, Params &p, const ClearList &cl, F &&enqueue) {
  uint64_t key[3];
  launch_shape(p, key);
  rtm_ctx::GraphEntry *hit = nullptr;
  for (auto &e : c->graphs)
    if (e.gen == c->gen && e.key[0] == key[0] && e.key[1] == key[1] && e.key[2] == key[2]) hit = &e;
  if (!hit) {
    if (!c->graphs.empty() && c->graphs.front().gen != c->gen) graphs_clear(c);  // stale pointers
    // Captured on a private non-blocking stream (capture is not permitted on the legacy default
    // stream, which the context stream may be); replayed on the context stream.
    if (!c->cap_st) CK(cudaStreamCreateWithFlags(&c->cap_st, cudaStreamNonBlocking));
    cudaGraph_t g = nullptr;
    cudaStream_t user = c->st;
    cudaError_t ce = cudaStreamBeginCapture(c->cap_st, cudaStreamCaptureModeThreadLocal);
    rtm_status s = RTM_OK;
    if (ce == cudaSuccess) {
      c->st = c->cap_st;
      s = enqueue();
      c->st = user;
      ce = cudaStreamEndCapture(c->cap_st, &g);
    }
    if (s) {
      if (g) cudaGraphDestroy(g);
      return s;
    }
    cudaGraphExec_t x = nullptr;
    if (ce != cudaSuccess || !g || cudaGraphInstantiate(&x, g, 0) != cudaSuccess) {
      cudaGetLastError();  // capture of this sequence unsupported here: launch directly from now on
      if (g) cudaGraphDestroy(g);
      c->graph_broken = true;
      return enqueue();
    }
    rtm_ctx::GraphEntry e;
    memcpy(e.key, key, sizeof(key));
    e.gen = c->gen;
    e.g = g;
    e.x = x;
    size_t n = 0;
    CK(cudaGraphGetNodes(g, nullptr, &n));
    std::vector<cudaGraphNode_t> nodes(n);
    CK(cudaGraphGetNodes(g, nodes.data(), &n));
    for (cudaGraphNode_t nd : nodes) {
      cudaGraphNodeType t;
      CK(cudaGraphNodeGetType(nd, &t));
      if (t != cudaGraphNodeTypeKernel) continue;
      cudaKernelNodeParams kp;
      CK(cudaGraphKernelNodeGetParams(nd, &kp));
      kp.kernelParams = nullptr;
      kp.extra = nullptr;
      e.kn.push_back(nd);
      e.kp.push_back(kp);
    }
    if (c->graphs.size() >= kGraphCacheSize) {  // evict the least recently used shape
      size_t lru = 0;
      for (size_t i = 1; i < c->graphs.size(); ++i)
        if (c->graphs[i].used < c->graphs[lru].used) lru = i;
      graph_free(c->graphs[lru]);
      c->graphs.erase(c->graphs.begin() + (long)lru);
    }
    c->graphs.push_back(std::move(e));
    hit = &c->graphs.back();  // captured with this call's arguments: launch as is
    ++c->graph_captures;
  } else {
    void *a1[] = {&p};
    ClearList cc = cl;
    long long *Bs = (long long *)c->Bs.p, *Be = (long long *)c->Be.p;
    void *a4[] = {&p, &cc, &Bs, &Be};
    const void *prep = prep_kernel_fn();
    for (size_t i = 0; i < hit->kn.size(); ++i) {
      cudaKernelNodeParams kp = hit->kp[i];
      kp.kernelParams = kp.func == prep ? a4 : a1;
      CK(cudaGraphExecKernelNodeSetParams(hit->x, hit->kn[i], &kp));
    }
    count_launches((unsigned)hit->kn.size());
    ++c->graph_replays;
  }
  hit->used = ++c->graph_tick;
  CK(cudaGraphLaunch(hit->x, c->st));
  return RTM_OK;
}

rtm_status reduce_local(rtm_ctx *c, const int64_t *t_end, uint32_t W, Params &p) {
  if (c->sticky) return (rtm_status)c->sticky;
  if (c->merge_pending) return RTM_E_STATE;  // the previous local reduce awaits rtm_merge
  if (!t_end || W == 0) return RTM_E_INVALID;
  if (t_end[0] < c->t_prev) return RTM_E_INVALID;
  const int64_t max_wlen = max_window_len(c->bin_log);
  if (t_end[0] - c->t_prev >= max_wlen) return RTM_E_INVALID;
  for (uint32_t w = 1; w < W; ++w)
    if (t_end[w] < t_end[w - 1] || t_end[w] - t_end[w - 1] >= max_wlen) return RTM_E_INVALID;
  CK(cudaSetDevice(c->device));

  const void *sp, *ep;
  uint64_t ns, ne;
  pending(c->s_dev, c->s_own, c->s_own_n, &sp, &ns);
  pending(c->e_dev, c->e_own, c->e_own_n, &ep, &ne);

  rtm_status s;
  // ---- window bounds T[0..W] and split positions
  if ((s = ensure(c, c->T, (size_t)(W + 1) * 8))) return s;
  if ((s = ensure(c, c->Bs, (size_t)(W + 3) * 8))) return s;
  if ((s = ensure(c, c->Be, (size_t)(W + 3) * 8))) return s;
  if ((s = ensure(c, c->rts, (size_t)(W + 3) * 4))) return s;
  if ((s = ensure(c, c->rte, (size_t)(W + 3) * 4))) return s;
  const size_t small = (size_t)(W + 1) * 8;
  if ((s = ensure_pinned(c, c->h_small, small))) return s;
  long long *hT = (long long *)c->h_small.p;
  hT[0] = c->t_prev;
  for (uint32_t w = 0; w < W; ++w) hT[w + 1] = t_end[w];

  memset(&p, 0, sizeof(p));
  p.nb = c->nb; p.nc = c->nc; p.nk = c->nk; p.nbins = c->nbins; p.ncw = c->ncw; p.k = c->k;
  p.bin_log = c->bin_log;
  // Few-unit calls (fewer (window, bin) units than SMs: one-window streaming calls on a C2-sized
  // registry) fold 128-buffer bins: twice the units, half the chain per unit.
  if (p.bin_log == 8 && (uint64_t)W * p.nbins < (uint64_t)c->n_sms && ((c->nb + 127) >> 7) <= kLmMaxBins) {
    p.bin_log = 7;
    p.nbins = (c->nb + 127) >> 7;
  }
  const uint32_t nbins = p.nbins;
  p.rank_mode = c->rank_mode; p.H = c->H; p.hang_mode = c->hang_mode;
  p.cap = (const uint16_t *)c->cap.p; p.owner = (const uint32_t *)c->owner.p;
  p.elig = (const uint8_t *)c->elig.p; p.ktotal = (const int64_t *)c->ktotal.p;
  p.klive = (const uint8_t *)c->klive.p;
  p.all_live = std::find(c->klive_h.begin(), c->klive_h.end(), (uint8_t)0) == c->klive_h.end();
  p.rcp = (const unsigned long long *)c->rcp.p; p.elig_ids = (const uint32_t *)c->elig_ids.p; p.n_elig = c->n_elig;
  // A fresh look-back epoch for every call, taken before any kernel runs: a call that failed
  // after its fold published flags (order error, exchange error) must not leave flags that
  // the next call would read as already published.
  c->epoch = c->epoch == 0xFFFFFFFFu ? 1u : c->epoch + 1u;
  p.W = W; p.epoch = c->epoch;
  p.narrow = 1;
  int64_t wlen_max = 0;
  for (uint32_t w = 0; w < W; ++w) {
    const int64_t len = t_end[w] - (w ? t_end[w - 1] : c->t_prev);
    wlen_max = std::max(wlen_max, len);
    if (len >= ((int64_t)1 << 32)) p.narrow = 0;
  }
  // the fold's integral term D lies in [0, cap * Wlen]: 32 bits when that is < 2^32
  p.narrow_d = p.narrow && (uint64_t)c->cap_max * (uint64_t)wlen_max < ((uint64_t)1 << 32);
  if (c->rank_mode == RTM_RANK_MEAN && !p.narrow) return RTM_E_INVALID;  // before any launch
  p.T = (const long long *)c->T.p;
  if (W + 1 <= kTInline) {
    p.t_inline = 1;
    for (uint32_t w = 0; w <= W; ++w) p.Tin[w] = hT[w];
  }
  p.s = (const rtm_level_sample *)sp; p.ns = ns;
  p.e = (const rtm_task_event *)ep; p.ne = ne;

  p.Bs = (const long long *)c->Bs.p; p.Be = (const long long *)c->Be.p;
  p.rts = (const uint32_t *)c->rts.p; p.rte = (const uint32_t *)c->rte.p;
  // tile-count upper bounds: every region adds at most one partial tile
  const uint32_t nts = (uint32_t)((ns + kTileS - 1) / kTileS) + W + 2;
  const uint32_t nte = (uint32_t)((ne + kTileE - 1) / kTileE) + W + 2;

  // ---- workspaces
  const size_t Wn = W;
  if ((s = ensure(c, c->treg_s, (size_t)nts * 4))) return s;
  if ((s = ensure(c, c->treg_e, (size_t)nte * 4))) return s;
  if ((s = ensure(c, c->tdesc, (size_t)nts * sizeof(TileDesc)))) return s;
  if ((s = ensure(c, c->soff, (size_t)nts * (nbins + 1) * 2))) return s;
  if ((s = ensure(c, c->stage, (size_t)nts * kTileS * 8))) return s;
  // more than 170 bins: two-pass partition (superbins, then bins per (window, superbin))
  const bool two_pass = partition_two_pass(nbins, p.narrow != 0);
  if (two_pass) {
    if ((s = ensure(c, c->stage2, (size_t)nts * kTileS * 8))) return s;
    if ((s = ensure(c, c->woff, (size_t)W * (nbins + 1) * 4))) return s;
  }
  if ((s = ensure(c, c->smeta, (size_t)nts * sizeof(TileMeta)))) return s;
  if ((s = ensure(c, c->emeta, (size_t)nte * sizeof(TileMeta)))) return s;
  if ((s = ensure(c, c->lastlvl, Wn * c->nb * 2))) return s;
  if (c->flags.cap < Wn * nbins * 4) {
    if ((s = ensure(c, c->flags, Wn * nbins * 4, true))) return s;
  }
  if ((s = ensure(c, c->res, res_layout(c, W).bytes))) return s;
  if ((s = ensure(c, c->kdelta, Wn * c->nk * 2 * 4))) return s;
  // per-component event deltas: zeroed at allocation and by rtm_reset, re-zeroed by k_progress
  // after it folds them into the cumulative counts (no per-call clear: C5 1.3 MB)
  if ((s = ensure(c, c->cdelta, (size_t)c->nc * 2 * 8, true))) return s;
  if ((s = ensure(c, c->active, Wn * c->ncw * 4))) return s;
  if ((s = ensure(c, c->anyfull, Wn * c->ncw * 4))) return s;
  if ((s = ensure(c, c->hung, Wn * c->ncw * 4))) return s;
  if (hang_block_path(W, c->H)) {
    if ((s = ensure(c, c->hsfx, Wn * c->ncw * 4))) return s;
  }
  if ((s = ensure(c, c->unit_ctr, 16))) return s;
  if ((s = ensure(c, c->bstat, (size_t)c->nb * sizeof(rtm_buffer_stat)))) return s;
  if (c->rank_mode == RTM_RANK_MEAN) {  // order keys (windows shorter than 2^32 ticks, checked above)
    if ((s = ensure(c, c->mkey, Wn * c->nb * 8))) return s;
    p.mkey = (unsigned long long *)c->mkey.p;
    p.rcp64 = (const unsigned long long *)c->rcp64.p;
    if (c->world > 1) {  // the merge ranks the ranks' candidates by these keys
      if ((s = ensure(c, c->tkey, Wn * c->k * 8))) return s;
      p.tkey = (unsigned long long *)c->tkey.p;
    }
  }
  p.persist = (uint32_t *)c->persist.p;
  p.tk_slices = topk_slices(c->nb, c->k, W, c->n_sms, c->n_elig == c->nb && c->rank_mode != RTM_RANK_MEAN,
                            &p.tk_slice_len);
  if (p.tk_slices > 1) {
    if ((s = ensure(c, c->tkscr, (size_t)W * p.tk_slices * c->k * 8))) return s;
    p.tk_scratch = (unsigned long long *)c->tkscr.p;
  }
  if ((s = ensure(c, c->comps, (size_t)c->nc * sizeof(rtm_component_tasks)))) return s;
  // Very sparse calls on the two-pass path (C5): the sequential fold walks the windows of a bin in
  // seq_ranges ranges at once, so ~2 warps per SM slot instead of one per bin (C5: 2560 bins).
  size_t endkey_bytes = 0;
  {
    Params q = p;
    q.ns = ns;
    if (two_pass && fold_sequential(q) && W >= 128) {
      const uint32_t want = (uint32_t)((2u * (uint32_t)c->n_sms * 24u + nbins - 1) / nbins);
      uint32_t R = std::min<uint32_t>({want, 8u, W / 64u});
      if (R > 1) {
        p.seq_range_len = (W + R - 1) / R;
        R = (W + p.seq_range_len - 1) / p.seq_range_len;
      }
      if (R > 1) {
        p.seq_ranges = R;
        endkey_bytes = (size_t)(R - 1) * c->nb * 8;
        if ((s = ensure(c, c->endkey, endkey_bytes))) return s;
        p.endkey = (unsigned long long *)c->endkey.p;
      }
    }
  }

  ClearList prep_cl;
  {
    const ResLayout L = res_layout(c, W);
    ClearList cl;
    cl.add(c->res.p, (size_t)kWinFields * Wn * 8);
    cl.add((char *)c->res.p + L.status, 16);
    cl.add(c->kdelta.p, Wn * c->nk * 2 * 4);
    cl.add(c->active.p, Wn * c->ncw * 4);
    cl.add(c->anyfull.p, Wn * c->ncw * 4);
    // long H, call shorter than H: the hang kernel stops at the first window its prefix AND empties
    if (c->H > 64 && W < c->H) cl.add(c->hung.p, Wn * c->ncw * 4);
    cl.add(c->unit_ctr.p, 16);
    if (endkey_bytes) cl.add(c->endkey.p, endkey_bytes);
    prep_cl = cl;
  }

  p.tdesc = (TileDesc *)c->tdesc.p; p.tile_reg_s = (const uint32_t *)c->treg_s.p; p.tile_reg_e = (const uint32_t *)c->treg_e.p;
  p.n_tiles_s = nts; p.n_tiles_e = nte;
  p.soff = (uint16_t *)c->soff.p; p.stage = (unsigned long long *)c->stage.p;
  if (two_pass) {
    p.nsb = (c->nb + (1u << kSupLog) - 1) >> kSupLog;
    p.stage2 = (unsigned long long *)c->stage2.p;
    p.woff = (uint32_t *)c->woff.p;
  }
  p.smeta = (TileMeta *)c->smeta.p; p.emeta = (TileMeta *)c->emeta.p;
  p.lastlvl = (uint16_t *)c->lastlvl.p; p.flags = (uint32_t *)c->flags.p;
  set_result_ptrs(c, W, p);
  p.kdelta = (uint32_t *)c->kdelta.p;
  p.cdelta = (unsigned long long *)c->cdelta.p; p.active = (uint32_t *)c->active.p;
  p.anyfull = (uint32_t *)c->anyfull.p; p.hung = (uint32_t *)c->hung.p;
  p.hsfx = hang_block_path(W, c->H) ? (uint32_t *)c->hsfx.p : nullptr;
  p.unit_ctr = (uint32_t *)c->unit_ctr.p;
  p.carry_in = (const uint16_t *)c->carry[c->cur].p; p.carry_out = (uint16_t *)c->carry[c->cur ^ 1].p;
  p.run = (const uint32_t *)c->run[c->cur].p;
  p.run_out = (uint32_t *)c->run[c->cur ^ 1].p;
  p.kstart = (long long *)c->kstart.p; p.kend = (long long *)c->kend.p;
  p.cstart = (long long *)c->cstart.p; p.cend = (long long *)c->cend.p;
  p.bstat = (rtm_buffer_stat *)c->bstat.p;
  p.gid = (const uint32_t *)c->gid.p; p.n_global = c->n_global; p.pack_nb = c->pack_nb;
  p.bstat_g = (rtm_buffer_stat *)c->bstat_g.p;
  p.comps = (rtm_component_tasks *)c->comps.p;

#ifdef RTM_PHASE_TIMING
  static unsigned long long *dbg = nullptr;
  if (!dbg) cudaMalloc(&dbg, 64);
  cudaMemsetAsync(dbg, 0, 64, c->st);
  p.dbg = dbg;
#endif
  // Task events are independent of the sample path.  Lane-major partition path: the persistent
  // partition kernel runs the event tiles after its sample tiles (claimed dynamically), so no
  // concurrent kernel competes with the issue-bound fold.  Otherwise: a side stream, overlapped
  // with the partition and the fold, joined before the kernels that read the event outputs.
  p.fuse_events = partition_fuses_events(p.nbins, nts, two_pass) ? 1 : 0;
  p.persist_inline = c->world == 1 && p.persist;  // the top-k kernels count their winners (world 1)
  // The launch sequence (every kernel takes this call's Params by value; k_prep also the clear
  // list and the split buffers).  Direct launches, or captured once per launch shape into a CUDA
  // graph and replayed (rtm_use_graphs).
  auto enqueue = [&]() -> rtm_status {
  if (!p.t_inline) CK(cudaMemcpyAsync(c->T.p, hT, (size_t)(W + 1) * 8, cudaMemcpyHostToDevice, c->st));
  // clear the call's accumulators, region boundaries, tile tables: one cooperative launch
  LAUNCH(KT_SPLIT, 0,
         launch_prep(p, prep_cl, (long long *)c->Bs.p, (long long *)c->Be.p, c->n_sms, c->st));
  CK(cudaGetLastError());
  if (!p.fuse_events) {
    CK(cudaEventRecord(c->ev_fork, c->st));
    CK(cudaStreamWaitEvent(c->st2, c->ev_fork, 0));
    if (c->prof) prof_begin_on(c, KT_EVENTS, (uint64_t)ne * 16, c->st2);
    launch_events(p, c->st2);
    if (c->prof) prof_end_on(c, c->st2);
    CK(cudaEventRecord(c->ev_join, c->st2));
  }
  // algorithmic bytes: 16 B per record, read once - charged to
  // the kernel that reads the records (the partition, + the event tiles it runs when fused); the
  // 8-B staging entries between partition and fold are not algorithmic (ncu traffic shows them)
  LAUNCH(KT_PARTITION, (uint64_t)ns * 16 + (p.fuse_events ? (uint64_t)ne * 16 : 0),
         launch_partition(p, c->n_sms, c->st));
  // The order check (tile metadata) and the progress bars (event counts) do not read the fold's
  // outputs: on the side stream, beside the fold (after the event kernel when it runs there);
  // joined before the top-k.  One-window streaming calls: -13 us of dependent launches.
  constexpr bool side = true;  // measured: C2 step 1.575 -> 1.556 ms
  if (side) {
    CK(cudaEventRecord(c->ev_fork, c->st));
    CK(cudaStreamWaitEvent(c->st2, c->ev_fork, 0));
    if (c->prof) prof_begin_on(c, KT_ORDER, 0, c->st2);
    launch_order_check(p, c->st2);
    if (c->prof) prof_end_on(c, c->st2);
    if (c->prof) prof_begin_on(c, KT_PROGRESS, 0, c->st2);
    launch_progress(p, c->st2);
    if (c->prof) prof_end_on(c, c->st2);
    CK(cudaEventRecord(c->ev_join, c->st2));
  }
  if (p.nsb) LAUNCH(KT_SUBPART, 0, launch_subpart(p, c->n_sms, c->st));
  LAUNCH(KT_FOLD, 0, launch_fold(p, c->n_sms, c->st));
  if (side || !p.fuse_events) CK(cudaStreamWaitEvent(c->st, c->ev_join, 0));
  if (!side) LAUNCH(KT_ORDER, 0, launch_order_check(p, c->st));
  // the hang flags (fold's anyfull + event activity bits) and the top-k (fold's last levels) are
  // independent: the hang kernel on the side stream beside the top-k (the waits above are already
  // enqueued, so the fork / join events can be recorded again)
  constexpr bool side_hang = true;  // measured: C2 step 1.559 -> 1.552 ms
  if (side_hang) {
    CK(cudaEventRecord(c->ev_fork, c->st));
    CK(cudaStreamWaitEvent(c->st2, c->ev_fork, 0));
    if (c->prof) prof_begin_on(c, KT_HANG, 0, c->st2);
    launch_hang(p, c->st2);
    if (c->prof) prof_end_on(c, c->st2);
    CK(cudaEventRecord(c->ev_join, c->st2));
  }
  LAUNCH(KT_TOPK, 0, launch_topk(p, c->st));  // world > 1: persistence counted from the merged lists
  if (side_hang) CK(cudaStreamWaitEvent(c->st, c->ev_join, 0));
  else LAUNCH(KT_HANG, 0, launch_hang(p, c->st));
  if (!side) LAUNCH(KT_PROGRESS, 0, launch_progress(p, c->st));
  CK(cudaGetLastError());
  return RTM_OK;
  };
  if (graph_use(c, W)) s = graph_launch(c, p, prep_cl, enqueue);
  else s = enqueue();
  p.persist_inline = 0;
  if (s) return s;
#ifdef RTM_PHASE_TIMING
  {
    unsigned long long h[8];
    cudaMemcpyAsync(h, p.dbg, 64, cudaMemcpyDeviceToHost, c->st);
    cudaStreamSynchronize(c->st);
    fprintf(stderr, "[lookback] units=%llu steps=%llu (%.2f / unit) spins=%llu\n", (unsigned long long)W * p.nbins,
            h[0], (double)h[0] / ((double)W * p.nbins), h[6]);
    if (h[7])
      fprintf(stderr, "[phase] tiles=%llu  -=%.0f wait_raw=%.0f scan=%.0f rank=%.0f B1=%.0f bases+scatter=%.0f -=%.0f (cycles/tile, thread 0)\n",
              h[7], (double)h[0] / h[7], (double)h[1] / h[7], (double)h[2] / h[7], (double)h[3] / h[7],
              (double)h[4] / h[7], (double)h[5] / h[7], (double)h[6] / h[7]);
  }
#endif
  return RTM_OK;
}

// D2H of the per-window results and bookkeeping after a (local or merged) reduce.
rtm_status finish(rtm_ctx *c, const int64_t *t_end, uint32_t W, rtm_window_summary *out) {
  const size_t Wn = W;
  const ResLayout L = res_layout(c, W);
  const size_t bytes = L.bytes;
  rtm_status s;
  if ((s = ensure_pinned(c, c->h_res, bytes))) return s;
  char *h = (char *)c->h_res.p;
  unsigned long long *hwin = (unsigned long long *)(h + L.win);
  unsigned long long *htopk = (unsigned long long *)(h + L.topk);
  long long *hprog = (long long *)(h + L.prog);
  uint32_t *htopk_n = (uint32_t *)(h + L.topk_n);
  uint32_t *hstatus = (uint32_t *)(h + L.status);
  // one copy: the device results buffer has the same layout (res_layout)
  CK(cudaMemcpyAsync(h, c->res.p, bytes, cudaMemcpyDeviceToHost, c->st));
  CK(cudaStreamSynchronize(c->st));
  prof_collect(c);
  if (*hstatus & 4u) {  // look-back wait timed out: internal error, never expected
    c->sticky = RTM_E_CUDA;
    return RTM_E_CUDA;
  }
  if (*hstatus) {
    c->sticky = RTM_E_ORDER;
    return RTM_E_ORDER;
  }
  c->sum.resize(Wn);
  c->t_end_h.assign(t_end, t_end + W);
  for (uint32_t w = 0; w < W; ++w) {
    rtm_window_summary &S = c->sum[w];
    S.t_begin = w ? t_end[w - 1] : c->t_prev;
    S.t_end = t_end[w];
    S.n_samples = hwin[WF_SAMPLES * Wn + w];
    S.n_events = hwin[WF_EVENTS * Wn + w];
    S.n_dropped = hwin[WF_DROPPED * Wn + w];
    S.digest = hwin[WF_DIGEST * Wn + w];
    S.n_touched = (uint32_t)hwin[WF_TOUCHED * Wn + w];
    S.n_hung = (uint32_t)hwin[WF_HUNG * Wn + w];
  }
  if (c->n_watch) {  // value monitor: append this batch's points to the rings
    const rtm_buffer_stat *hw = (const rtm_buffer_stat *)(h + L.watch);
    for (uint32_t q = 0; q < c->n_watch; ++q) {
      if (c->watch_local[q] == 0xFFFFFFFFu) continue;
      std::vector<rtm_watch_point> &r = c->ring[q];
      if (r.size() != RTM_WATCH_POINTS) r.assign(RTM_WATCH_POINTS, rtm_watch_point());
      for (uint32_t w = 0; w < W; ++w) {
        rtm_watch_point &pt = r[(c->ring_head[q] + c->ring_n[q]) % RTM_WATCH_POINTS];
        pt.t_end = t_end[w];
        pt.stat = hw[(size_t)w * RTM_WATCH_MAX + q];
        if (c->ring_n[q] < RTM_WATCH_POINTS) ++c->ring_n[q];
        else c->ring_head[q] = (c->ring_head[q] + 1) % RTM_WATCH_POINTS;
      }
    }
  }
  c->topk_h = htopk;
  c->topk_n_h = htopk_n;
  c->prog_h = reinterpret_cast<const rtm_progress_entry *>(hprog);
  if (out) memcpy(out, c->sum.data(), Wn * sizeof(rtm_window_summary));
  c->t_prev = t_end[W - 1];
  c->cur ^= 1;
  c->merge_pending = false;
  c->have = true;
  c->W = W;
  c->s_dev.clear();
  c->e_dev.clear();
  c->s_own_n = c->e_own_n = 0;
  return RTM_OK;
}

}  // namespace

// ================================================================================================
extern "C" {

const char *rtm_status_str(rtm_status s) {
  switch (s) {
    case RTM_OK: return "ok";
    case RTM_E_INVALID: return "invalid argument";
    case RTM_E_CUDA: return "CUDA error";
    case RTM_E_COMM: return "cross-rank exchange failed";
    case RTM_E_ORDER: return "field-valid records not non-decreasing in ts";
    case RTM_E_TOO_SMALL: return "output capacity too small";
    case RTM_E_STATE: return "call not valid in the current state";
    case RTM_E_NOMEM: return "device allocation failed";
  }
  return "unknown status";
}

const char *rtm_version(void) { return "librtm 0.1 sm_100a (window-snapshot reducer)"; }

uint64_t rtm_kernel_launches(void) { return (uint64_t)kernel_launches(); }

rtm_status rtm_create(const rtm_config *cfg, rtm_ctx **out) {
  if (!cfg || !out) return RTM_E_INVALID;
  *out = nullptr;
  if (cfg->n_buffers == 0 || cfg->n_buffers > (uint32_t)kMaxBins * kBin) return RTM_E_INVALID;
  if (cfg->n_components == 0 || cfg->n_components > (1u << 20)) return RTM_E_INVALID;
  if (cfg->n_kernels == 0 || cfg->n_kernels > 2048) return RTM_E_INVALID;
  if (cfg->k == 0 || cfg->k > 1024 || cfg->hang_windows == 0) return RTM_E_INVALID;
  if (cfg->rank_mode != RTM_RANK_PERCENT && cfg->rank_mode != RTM_RANK_SIZE && cfg->rank_mode != RTM_RANK_MEAN)
    return RTM_E_INVALID;
  if (cfg->hang_mode != RTM_HANG_FULL && cfg->hang_mode != RTM_HANG_NONEMPTY) return RTM_E_INVALID;
  if (!cfg->buffer_owner || !cfg->buffer_capacity || !cfg->kernel_total) return RTM_E_INVALID;
  if (cfg->world < 1 || cfg->rank < 0 || cfg->rank >= cfg->world) return RTM_E_INVALID;
  for (uint32_t b = 0; b < cfg->n_buffers; ++b)
    if (cfg->buffer_capacity[b] == 0 || cfg->buffer_capacity[b] == 0xFFFFu || cfg->buffer_owner[b] >= cfg->n_components)
      return RTM_E_INVALID;
  if (cfg->buffer_global_id) {  // strictly increasing global ids below n_global_buffers
    for (uint32_t b = 0; b < cfg->n_buffers; ++b)
      if (cfg->buffer_global_id[b] >= cfg->n_global_buffers || (b && cfg->buffer_global_id[b] <= cfg->buffer_global_id[b - 1]))
        return RTM_E_INVALID;
  }
  if (cfg->pack_buffers && cfg->pack_buffers < cfg->n_buffers) return RTM_E_INVALID;
  if (cfg->world > 1 && !merge_fits(cfg->world, cfg->k)) return RTM_E_INVALID;  // merge candidates in smem
  int ndev = 0;
  if (cudaGetDeviceCount(&ndev) != cudaSuccess || cfg->device < 0 || cfg->device >= ndev) {
    cudaGetLastError();
    return RTM_E_INVALID;
  }
  rtm_ctx *c = new rtm_ctx();
  c->nb = cfg->n_buffers;
  c->nc = cfg->n_components;
  c->nk = cfg->n_kernels;
  // 256 buffers per bin; 128 for large registries (131073 .. 524288 buffers, e.g. C5's 327680):
  // very sparse windows are folded by one warp per bin walking the windows in order, and halving
  // the bin doubles the warps (the partition fallback takes up to 4096 bins)
  c->bin_log = (c->nb > 131072u && c->nb <= kMaxBins * 128u) ? 7 : 8;
#ifdef RTM_FORCE_BIN_LOG  // compile-time A/B builds only (tools/build_variant.sh)
  c->bin_log = RTM_FORCE_BIN_LOG;
  if (c->nb > kMaxBins * (1u << c->bin_log)) c->bin_log = 8;
#endif
  c->nbins = (c->nb + (1u << c->bin_log) - 1) >> c->bin_log;
  c->ncw = (c->nc + 31) / 32;
  c->k = cfg->k;
  c->H = cfg->hang_windows;
  c->rank_mode = cfg->rank_mode;
  c->hang_mode = cfg->hang_mode;
  c->device = cfg->device;
  c->rank = cfg->rank;
  c->world = cfg->world;
  c->t0 = cfg->t0;
  c->t_prev = cfg->t0;
  c->n_global = cfg->buffer_global_id ? cfg->n_global_buffers : 0;
  if (cfg->buffer_global_id) c->gid_h.assign(cfg->buffer_global_id, cfg->buffer_global_id + c->nb);
  c->pack_nb = cfg->pack_buffers ? cfg->pack_buffers : cfg->n_buffers;
  c->allgather = cfg->allgather;
  c->allgather_user = cfg->allgather_user;
  c->ag_on_stream = cfg->allgather_on_stream != 0;
  c->st = (cudaStream_t)cfg->stream;
  if (cudaSetDevice(c->device) != cudaSuccess) { cudaGetLastError(); delete c; return RTM_E_CUDA; }
  configure_kernels_once();
  cudaDeviceGetAttribute(&c->n_sms, cudaDevAttrMultiProcessorCount, c->device);
  // side stream at the highest priority: its small kernels (order check, progress) are dispatched
  // before the persistent fold's CTAs, which would otherwise hold every SM until the fold ends
  int prio_lo = 0, prio_hi = 0;
  cudaDeviceGetStreamPriorityRange(&prio_lo, &prio_hi);
  if (cudaStreamCreateWithPriority(&c->st2, cudaStreamNonBlocking, prio_hi) != cudaSuccess ||
      cudaEventCreateWithFlags(&c->ev_fork, cudaEventDisableTiming) != cudaSuccess ||
      cudaEventCreateWithFlags(&c->ev_join, cudaEventDisableTiming) != cudaSuccess) {
    cudaGetLastError();
    delete c;
    return RTM_E_CUDA;
  }
  rtm_status s = RTM_OK;
  auto fail = [&](rtm_status e) { rtm_destroy(c); return e; };
  if ((s = ensure(c, c->cap, (size_t)c->nb * 2)) || (s = ensure(c, c->owner, (size_t)c->nb * 4)) ||
      (s = ensure(c, c->elig, (size_t)c->nb)) || (s = ensure(c, c->ktotal, (size_t)c->nk * 8)) ||
      (s = ensure(c, c->carry[0], (size_t)c->nb * 2)) || (s = ensure(c, c->carry[1], (size_t)c->nb * 2)) ||
      (s = ensure(c, c->run[0], (size_t)c->nc * 4)) || (s = ensure(c, c->run[1], (size_t)c->nc * 4)) ||
      (s = ensure(c, c->kstart, (size_t)c->nk * 8)) ||
      (s = ensure(c, c->kend, (size_t)c->nk * 8)) || (s = ensure(c, c->cstart, (size_t)c->nc * 8)) ||
      (s = ensure(c, c->cend, (size_t)c->nc * 8)) || (s = ensure(c, c->rcp, (size_t)65536 * 8)) ||
      (s = ensure(c, c->elig_ids, (size_t)c->nb * 4)) ||
      (s = ensure(c, c->persist, (size_t)(c->n_global ? c->n_global : c->nb) * 4)) ||
      (s = ensure(c, c->klive, (size_t)c->nk)) || (s = ensure(c, c->gcum, (size_t)c->nk * 16)))
    return fail(s);
  c->ktotal0.assign(cfg->kernel_total, cfg->kernel_total + c->nk);
  for (uint32_t b = 0; b < c->nb; ++b) c->cap_max = std::max<uint32_t>(c->cap_max, cfg->buffer_capacity[b]);
  if (c->rank_mode == RTM_RANK_MEAN) {
    if ((s = ensure(c, c->rcp64, (size_t)65536 * 8))) return fail(s);
    std::vector<unsigned long long> r64(65536, 0);
    for (uint32_t cc = 2; cc < 65536; ++cc) r64[cc] = (unsigned long long)(((unsigned __int128)1 << 64) / cc);
    if (cudaMemcpy(c->rcp64.p, r64.data(), 65536 * 8, cudaMemcpyHostToDevice) != cudaSuccess) {
      cudaGetLastError();
      return fail(RTM_E_CUDA);
    }
  }
  std::vector<uint8_t> elig(c->nb);
  std::vector<uint32_t> elig_ids;
  for (uint32_t b = 0; b < c->nb; ++b) {
    elig[b] = cfg->owned_components ? (cfg->owned_components[cfg->buffer_owner[b]] != 0) : 1;
    if (elig[b]) elig_ids.push_back(b);
  }
  c->n_elig = (uint32_t)elig_ids.size();
  c->elig_h = elig;
  std::vector<unsigned long long> rcp(65536, 0);
  for (uint32_t cc = 2; cc < 65536; ++cc) rcp[cc] = (1ull << 48) / cc;  // c == 1: only l == 0 < c
  if (cudaMemcpy(c->rcp.p, rcp.data(), 65536 * 8, cudaMemcpyHostToDevice) != cudaSuccess ||
      (c->n_elig && cudaMemcpy(c->elig_ids.p, elig_ids.data(), (size_t)c->n_elig * 4, cudaMemcpyHostToDevice) !=
                        cudaSuccess)) {
    cudaGetLastError();
    return fail(RTM_E_CUDA);
  }
  if (cudaMemcpy(c->cap.p, cfg->buffer_capacity, (size_t)c->nb * 2, cudaMemcpyHostToDevice) != cudaSuccess ||
      cudaMemcpy(c->owner.p, cfg->buffer_owner, (size_t)c->nb * 4, cudaMemcpyHostToDevice) != cudaSuccess ||
      cudaMemcpy(c->elig.p, elig.data(), (size_t)c->nb, cudaMemcpyHostToDevice) != cudaSuccess ||
      cudaMemcpy(c->ktotal.p, cfg->kernel_total, (size_t)c->nk * 8, cudaMemcpyHostToDevice) != cudaSuccess) {
    cudaGetLastError();
    return fail(RTM_E_CUDA);
  }
  if (cfg->buffer_global_id) {
    if ((s = ensure(c, c->gid, (size_t)c->nb * 4)) ||
        (s = ensure(c, c->bstat_g, (size_t)c->n_global * sizeof(rtm_buffer_stat))))
      return fail(s);
    if (cudaMemcpy(c->gid.p, cfg->buffer_global_id, (size_t)c->nb * 4, cudaMemcpyHostToDevice) != cudaSuccess ||
        cudaMemset(c->bstat_g.p, 0, (size_t)c->n_global * sizeof(rtm_buffer_stat)) != cudaSuccess) {
      cudaGetLastError();
      return fail(RTM_E_CUDA);
    }
  }
  if ((s = zero_state(c))) return fail(s);
  *out = c;
  return RTM_OK;
}

void rtm_destroy(rtm_ctx *c) {
  if (!c) return;
  cudaSetDevice(c->device);
  cudaStreamSynchronize(c->st);
  DevBuf *bufs[] = {&c->cap, &c->owner, &c->elig, &c->ktotal, &c->carry[0], &c->carry[1], &c->run[0], &c->run[1],
                    &c->kstart, &c->rcp, &c->elig_ids, &c->gid, &c->bstat_g,
                    &c->kend, &c->cstart, &c->cend, &c->flags, &c->s_own, &c->e_own, &c->T, &c->Bs, &c->Be,
                    &c->rts, &c->rte, &c->treg_s, &c->treg_e, &c->tdesc, &c->soff, &c->stage, &c->stage2, &c->woff, &c->smeta, &c->emeta,
                    &c->lastlvl, &c->res, &c->kdelta, &c->cdelta, &c->active, &c->anyfull, &c->hung,
                    &c->unit_ctr, &c->bstat, &c->comps, &c->pack,
                    &c->gathered, &c->tkscr, &c->mkey, &c->rcp64, &c->tkey, &c->persist, &c->klive,
                    &c->gcum, &c->tpack, &c->tgathered, &c->endkey, &c->hsfx};
  graphs_clear(c);
  if (c->cap_st) cudaStreamDestroy(c->cap_st);
  for (DevBuf *b : bufs) free_buf(*b);
  if (c->h_small.p) cudaFreeHost(c->h_small.p);
  if (c->h_res.p) cudaFreeHost(c->h_res.p);
  for (cudaEvent_t e : c->ev_pool) cudaEventDestroy(e);
  if (c->st2) cudaStreamSynchronize(c->st2), cudaStreamDestroy(c->st2);
  if (c->ev_fork) cudaEventDestroy(c->ev_fork);
  if (c->ev_join) cudaEventDestroy(c->ev_join);
  cudaGetLastError();
  delete c;
}

rtm_status rtm_reset(rtm_ctx *c) {
  if (!c) return RTM_E_INVALID;
  cudaSetDevice(c->device);
  cudaStreamSynchronize(c->st);
  cudaGetLastError();
  c->sticky = 0;
  for (uint32_t q = 0; q < RTM_WATCH_MAX; ++q) c->ring_head[q] = c->ring_n[q] = 0;
  return zero_state(c);
}

rtm_status rtm_bar_create(rtm_ctx *c, int64_t total, uint32_t *bar_id) {
  if (!c || !bar_id) return RTM_E_INVALID;
  if (c->sticky) return (rtm_status)c->sticky;
  uint32_t k = 0;
  while (k < c->nk && c->klive_h[k]) ++k;
  if (k == c->nk) return RTM_E_TOO_SMALL;
  CK(cudaSetDevice(c->device));
  const int64_t zero = 0;
  const uint8_t one = 1;
  CK(cudaMemcpyAsync((int64_t *)c->ktotal.p + k, &total, 8, cudaMemcpyHostToDevice, c->st));
  CK(cudaMemcpyAsync((int64_t *)c->kstart.p + k, &zero, 8, cudaMemcpyHostToDevice, c->st));
  CK(cudaMemcpyAsync((int64_t *)c->kend.p + k, &zero, 8, cudaMemcpyHostToDevice, c->st));
  CK(cudaMemcpyAsync((int64_t *)c->gcum.p + 2 * k, &zero, 8, cudaMemcpyHostToDevice, c->st));
  CK(cudaMemcpyAsync((int64_t *)c->gcum.p + 2 * k + 1, &zero, 8, cudaMemcpyHostToDevice, c->st));
  CK(cudaMemcpyAsync((uint8_t *)c->klive.p + k, &one, 1, cudaMemcpyHostToDevice, c->st));
  CK(cudaStreamSynchronize(c->st));  // pageable stack sources
  c->klive_h[k] = 1;
  c->bars_dirty = true;
  *bar_id = k;
  return RTM_OK;
}

rtm_status rtm_bar_update(rtm_ctx *c, uint32_t bar_id, int64_t total) {
  if (!c || bar_id >= c->nk || !c->klive_h[bar_id]) return RTM_E_INVALID;
  if (c->sticky) return (rtm_status)c->sticky;
  CK(cudaSetDevice(c->device));
  CK(cudaMemcpyAsync((int64_t *)c->ktotal.p + bar_id, &total, 8, cudaMemcpyHostToDevice, c->st));
  CK(cudaStreamSynchronize(c->st));
  c->bars_dirty = true;
  return RTM_OK;
}

rtm_status rtm_bar_destroy(rtm_ctx *c, uint32_t bar_id) {
  if (!c || bar_id >= c->nk || !c->klive_h[bar_id]) return RTM_E_INVALID;
  if (c->sticky) return (rtm_status)c->sticky;
  CK(cudaSetDevice(c->device));
  const uint8_t zero = 0;
  CK(cudaMemcpyAsync((uint8_t *)c->klive.p + bar_id, &zero, 1, cudaMemcpyHostToDevice, c->st));
  CK(cudaStreamSynchronize(c->st));
  c->klive_h[bar_id] = 0;
  c->bars_dirty = true;
  return RTM_OK;
}

rtm_status rtm_topk_persistence(rtm_ctx *c, uint32_t first, uint32_t count, uint32_t *out) {
  if (!c || (count && !out)) return RTM_E_INVALID;
  if (c->sticky) return (rtm_status)c->sticky;
  const uint32_t space = c->n_global ? c->n_global : c->nb;
  if ((uint64_t)first + count > space) return RTM_E_INVALID;
  if (!count) return RTM_OK;
  CK(cudaSetDevice(c->device));
  CK(cudaMemcpyAsync(out, (const uint32_t *)c->persist.p + first, (size_t)count * 4, cudaMemcpyDeviceToHost, c->st));
  CK(cudaStreamSynchronize(c->st));
  return RTM_OK;
}

rtm_status rtm_watch(rtm_ctx *c, const uint32_t *ids, uint32_t n) {
  if (!c || n > RTM_WATCH_MAX || (n && !ids)) return RTM_E_INVALID;
  if (c->merge_pending) return RTM_E_STATE;  // the pending merge copies results in the frozen layout
  const uint32_t space = c->gid.p ? c->n_global : c->nb;
  for (uint32_t q = 0; q < n; ++q) {
    if (ids[q] >= space) return RTM_E_INVALID;
    for (uint32_t r = 0; r < q; ++r)
      if (ids[r] == ids[q]) return RTM_E_INVALID;
  }
  for (uint32_t q = 0; q < n; ++q) {
    uint32_t loc = ids[q];
    if (!c->gid.p && !c->elig_h.empty() && !c->elig_h[loc]) loc = 0xFFFFFFFFu;  // owned by another rank
    if (c->gid.p) {  // rank-local numbering: the local buffer with this global id, if any
      auto it = std::lower_bound(c->gid_h.begin(), c->gid_h.end(), ids[q]);
      loc = (it != c->gid_h.end() && *it == ids[q]) ? (uint32_t)(it - c->gid_h.begin()) : 0xFFFFFFFFu;
    }
    c->watch_ids[q] = ids[q];
    c->watch_local[q] = loc;
  }
  c->n_watch = n;
  for (uint32_t q = 0; q < RTM_WATCH_MAX; ++q) c->ring_head[q] = c->ring_n[q] = 0;
  return RTM_OK;
}

rtm_status rtm_watch_series(rtm_ctx *c, uint32_t slot, rtm_watch_point *out, uint32_t *n_out) {
  if (!c || !out || !n_out || slot >= c->n_watch) return RTM_E_INVALID;
  const uint32_t n = c->ring_n[slot];
  for (uint32_t i = 0; i < n; ++i) out[i] = c->ring[slot][(c->ring_head[slot] + i) % RTM_WATCH_POINTS];
  *n_out = n;
  return RTM_OK;
}

rtm_status rtm_ingest(rtm_ctx *c, const rtm_level_sample *samples, uint64_t n_samples, const rtm_task_event *events,
                      uint64_t n_events, int32_t mem) {
  if (!c) return RTM_E_INVALID;
  if (c->sticky) return (rtm_status)c->sticky;
  if (mem != RTM_MEM_HOST && mem != RTM_MEM_DEVICE) return RTM_E_INVALID;
  if ((n_samples && !samples) || (n_events && !events)) return RTM_E_INVALID;
  if (mem == RTM_MEM_DEVICE && ((((uintptr_t)samples) & 15) || (((uintptr_t)events) & 15))) return RTM_E_INVALID;
  CK(cudaSetDevice(c->device));
  rtm_status s = append(c, c->s_dev, c->s_own, c->s_own_n, samples, n_samples, mem);
  if (s) return s;
  return append(c, c->e_dev, c->e_own, c->e_own_n, events, n_events, mem);
}

rtm_status rtm_window_reduce(rtm_ctx *c, const int64_t *t_end, uint32_t n_windows, rtm_window_summary *out) {
  if (!c) return RTM_E_INVALID;
  if (c->world > 1 && !c->allgather) return RTM_E_INVALID;
  Params p;
  rtm_status s = reduce_local(c, t_end, n_windows, p);
  if (s) return s;
  if (c->world > 1) {
    const uint64_t pb = pack_bytes(p);
    if ((s = ensure(c, c->pack, pb))) return s;
    if ((s = ensure(c, c->gathered, pb * c->world))) return s;
    launch_pack(p, c->pack.p, c->st);
    if (!c->ag_on_stream) CK(cudaStreamSynchronize(c->st));  // else the callback orders itself on st
    if (c->allgather(c->allgather_user, c->pack.p, c->gathered.p, pb) != 0) {
      c->sticky = RTM_E_COMM;
      return RTM_E_COMM;
    }
    LAUNCH(KT_MERGE, 0, launch_merge(p, c->gathered.p, c->world, (long long *)c->gcum.p, c->st));
    launch_persist(p, c->st);
    CK(cudaGetLastError());
    c->tables_synced = false;
  } else if (c->gid.p) {
    launch_scatter_bstat(p, c->st);
  }
  return finish(c, t_end, n_windows, out);
}

rtm_status rtm_window_reduce_local(rtm_ctx *c, const int64_t *t_end, uint32_t n_windows, const void **pack,
                                   uint64_t *pack_bytes_out) {
  if (!c || !pack || !pack_bytes_out) return RTM_E_INVALID;
  Params p;
  rtm_status s = reduce_local(c, t_end, n_windows, p);
  if (s) return s;
  const uint64_t pb = pack_bytes(p);
  if ((s = ensure(c, c->pack, pb))) return s;
  launch_pack(p, c->pack.p, c->st);
  CK(cudaGetLastError());  // the pack is complete in the context stream's order (no host sync)
  *pack = c->pack.p;
  *pack_bytes_out = pb;
  // remember the call for rtm_merge; no other reduce (and no rtm_watch, which would change the
  // results layout) until it runs
  c->t_end_h.assign(t_end, t_end + n_windows);
  c->W = n_windows;
  c->have = false;
  c->merge_pending = true;
  return RTM_OK;
}

rtm_status rtm_merge(rtm_ctx *c, const void *gathered, uint32_t world, rtm_window_summary *out) {
  if (!c || !gathered || world == 0) return RTM_E_INVALID;
  if (c->sticky) return (rtm_status)c->sticky;
  if (!c->merge_pending || c->t_end_h.empty() || c->have) return RTM_E_STATE;
  CK(cudaSetDevice(c->device));
  const uint32_t W = (uint32_t)c->t_end_h.size();
  Params p;
  memset(&p, 0, sizeof(p));
  p.nb = c->nb; p.nc = c->nc; p.nk = c->nk; p.nbins = c->nbins; p.ncw = c->ncw; p.k = c->k;
  p.rank_mode = c->rank_mode; p.W = W;
  p.ktotal = (const int64_t *)c->ktotal.p; p.rcp = (const unsigned long long *)c->rcp.p;
  p.klive = (const uint8_t *)c->klive.p;
  set_result_ptrs(c, W, p);
  p.hung = (uint32_t *)c->hung.p;
  p.comps = (rtm_component_tasks *)c->comps.p; p.bstat = (rtm_buffer_stat *)c->bstat.p;
  p.gid = (const uint32_t *)c->gid.p; p.n_global = c->n_global; p.pack_nb = c->pack_nb;
  p.bstat_g = (rtm_buffer_stat *)c->bstat_g.p;
  p.persist = (uint32_t *)c->persist.p;
  LAUNCH(KT_MERGE, 0, launch_merge(p, gathered, world, (long long *)c->gcum.p, c->st));
  launch_persist(p, c->st);
  CK(cudaGetLastError());
  c->tables_synced = c->world <= 1;
  std::vector<int64_t> te = c->t_end_h;
  return finish(c, te.data(), W, out);
}

// Params of the last call's tables (the on-demand exchange)
static Params table_params(rtm_ctx *c) {
  Params p;
  memset(&p, 0, sizeof(p));
  p.nb = c->nb; p.nc = c->nc; p.nk = c->nk; p.nbins = c->nbins; p.ncw = c->ncw; p.k = c->k;
  p.W = c->W;
  p.hung = (uint32_t *)c->hung.p;
  p.comps = (rtm_component_tasks *)c->comps.p; p.bstat = (rtm_buffer_stat *)c->bstat.p;
  p.cstart = (long long *)c->cstart.p; p.cend = (long long *)c->cend.p;
  p.gid = (const uint32_t *)c->gid.p; p.n_global = c->n_global; p.pack_nb = c->pack_nb;
  p.bstat_g = (rtm_buffer_stat *)c->bstat_g.p;
  return p;
}

rtm_status rtm_tables_local(rtm_ctx *c, const void **pack, uint64_t *bytes) {
  if (!c || !pack || !bytes) return RTM_E_INVALID;
  if (c->sticky) return (rtm_status)c->sticky;
  if (!c->have) return RTM_E_STATE;
  CK(cudaSetDevice(c->device));
  const Params p = table_params(c);
  const uint64_t tb = tables_bytes(p);
  rtm_status s;
  if ((s = ensure(c, c->tpack, tb))) return s;
  launch_pack_tables(p, c->tpack.p, c->st);
  CK(cudaGetLastError());  // complete in the context stream's order
  *pack = c->tpack.p;
  *bytes = tb;
  return RTM_OK;
}

rtm_status rtm_tables_merge(rtm_ctx *c, const void *gathered, uint32_t world) {
  if (!c || !gathered || world == 0) return RTM_E_INVALID;
  if (c->sticky) return (rtm_status)c->sticky;
  if (!c->have) return RTM_E_STATE;
  CK(cudaSetDevice(c->device));
  const Params p = table_params(c);
  launch_merge_tables(p, gathered, world, c->st);
  CK(cudaGetLastError());
  c->tables_synced = true;
  return RTM_OK;
}

rtm_status rtm_sync_tables(rtm_ctx *c) {
  if (!c) return RTM_E_INVALID;
  if (c->world > 1 && !c->allgather) return RTM_E_INVALID;
  if (c->world <= 1 || c->tables_synced) return c->sticky ? (rtm_status)c->sticky : (c->have ? RTM_OK : RTM_E_STATE);
  const void *pk;
  uint64_t tb;
  rtm_status s = rtm_tables_local(c, &pk, &tb);
  if (s) return s;
  if ((s = ensure(c, c->tgathered, tb * c->world))) return s;
  if (!c->ag_on_stream) CK(cudaStreamSynchronize(c->st));
  if (c->allgather(c->allgather_user, pk, c->tgathered.p, tb) != 0) {
    c->sticky = RTM_E_COMM;
    return RTM_E_COMM;
  }
  return rtm_tables_merge(c, c->tgathered.p, c->world);
}

uint64_t rtm_exchange_bytes(uint32_t n_windows, uint32_t k, uint32_t n_kernels, int32_t rank_mode) {
  return exchange_bytes(n_windows, k, n_kernels, rank_mode);
}

rtm_status rtm_topk_buffers(rtm_ctx *c, uint32_t window, rtm_topk_entry *out, uint32_t *n_out) {
  if (!c || !out || !n_out) return RTM_E_INVALID;
  if (c->sticky) return (rtm_status)c->sticky;
  if (!c->have) return RTM_E_STATE;
  if (window >= c->W) return RTM_E_INVALID;
  const uint32_t n = c->topk_n_h[window];
  for (uint32_t i = 0; i < c->k; ++i) {
    const unsigned long long e = c->topk_h[(size_t)window * c->k + i];
    out[i].buffer_id = i < n ? (uint32_t)(e & 0xFFFFFFFFu) : 0xFFFFFFFFu;
    out[i].level = i < n ? (uint16_t)((e >> 32) & 0xFFFFu) : 0;
    out[i].capacity = i < n ? (uint16_t)(e >> 48) : 0;
  }
  *n_out = n;
  return RTM_OK;
}

rtm_status rtm_window_results(rtm_ctx *c, uint32_t first, uint32_t count, rtm_window_summary *summaries,
                              rtm_topk_entry *topk, uint32_t *topk_n, rtm_progress_entry *bars) {
  if (!c) return RTM_E_INVALID;
  if (c->sticky) return (rtm_status)c->sticky;
  if (!c->have) return RTM_E_STATE;
  if ((uint64_t)first + count > c->W) return RTM_E_INVALID;
  if (summaries) memcpy(summaries, c->sum.data() + first, (size_t)count * sizeof(rtm_window_summary));
  if (topk_n) memcpy(topk_n, c->topk_n_h + first, (size_t)count * 4);
  if (bars)
    memcpy(bars, c->prog_h + (size_t)first * c->nk, (size_t)count * c->nk * sizeof(rtm_progress_entry));
  if (topk) {
    const unsigned long long *src = c->topk_h + (size_t)first * c->k;
    for (uint32_t w = 0; w < count; ++w) {
      const uint32_t n = c->topk_n_h[first + w];
      rtm_topk_entry *o = topk + (size_t)w * c->k;
      for (uint32_t i = 0; i < c->k; ++i) {
        const unsigned long long e = src[(size_t)w * c->k + i];
        o[i].buffer_id = i < n ? (uint32_t)(e & 0xFFFFFFFFu) : 0xFFFFFFFFu;
        o[i].level = i < n ? (uint16_t)((e >> 32) & 0xFFFFu) : 0;
        o[i].capacity = i < n ? (uint16_t)(e >> 48) : 0;
      }
    }
  }
  return RTM_OK;
}

rtm_status rtm_progress(rtm_ctx *c, uint32_t window, rtm_progress_entry *bars, rtm_component_tasks *comps) {
  if (!c || !bars) return RTM_E_INVALID;
  if (c->sticky) return (rtm_status)c->sticky;
  if (!c->have) return RTM_E_STATE;
  if (window >= c->W) return RTM_E_INVALID;
  if (comps && window != c->W - 1) return RTM_E_INVALID;
  if (comps && !c->tables_synced) return RTM_E_STATE;  // world > 1: rtm_sync_tables first
  memcpy(bars, c->prog_h + (size_t)window * c->nk, (size_t)c->nk * sizeof(rtm_progress_entry));
  if (comps) {
    CK(cudaSetDevice(c->device));
    CK(cudaMemcpyAsync(comps, c->comps.p, (size_t)c->nc * sizeof(rtm_component_tasks), cudaMemcpyDeviceToHost,
                       c->st));
    CK(cudaStreamSynchronize(c->st));
  }
  return RTM_OK;
}

// flagged component ids of `window` of the last batch, ascending
static rtm_status hung_list(rtm_ctx *c, uint32_t window, std::vector<uint32_t> &ids) {
  std::vector<uint32_t> bits(c->ncw);
  CK(cudaSetDevice(c->device));
  CK(cudaMemcpyAsync(bits.data(), (uint32_t *)c->hung.p + (size_t)window * c->ncw, (size_t)c->ncw * 4,
                     cudaMemcpyDeviceToHost, c->st));
  CK(cudaStreamSynchronize(c->st));
  ids.clear();
  for (uint32_t q = 0; q < c->ncw; ++q) {
    uint32_t x = bits[q];
    while (x) {
      const int bpos = __builtin_ctz(x);
      x &= x - 1;
      const uint32_t comp = q * 32 + bpos;
      if (comp < c->nc) ids.push_back(comp);
    }
  }
  return RTM_OK;
}

rtm_status rtm_hang_check(rtm_ctx *c, uint32_t window, uint32_t *comp_ids, uint32_t cap, uint32_t *n_hung) {
  if (!c || !n_hung || (cap && !comp_ids)) return RTM_E_INVALID;
  if (c->sticky) return (rtm_status)c->sticky;
  if (!c->have) return RTM_E_STATE;
  if (window >= c->W) return RTM_E_INVALID;
  if (!c->tables_synced) {  // world > 1: the merged count is known; the list needs the tables
    if (c->sum[window].n_hung == 0) {
      *n_hung = 0;
      return RTM_OK;
    }
    return RTM_E_STATE;
  }
  std::vector<uint32_t> ids;
  rtm_status s = hung_list(c, window, ids);
  if (s) return s;
  for (size_t i = 0; i < ids.size() && i < cap; ++i) comp_ids[i] = ids[i];
  *n_hung = (uint32_t)ids.size();
  return RTM_OK;
}

rtm_status rtm_set_links(rtm_ctx *c, const uint32_t *src, const uint32_t *dst, uint32_t n_links) {
  if (!c || (n_links && (!src || !dst))) return RTM_E_INVALID;
  for (uint32_t i = 0; i < n_links; ++i)
    if (src[i] >= c->nc || dst[i] >= c->nc) return RTM_E_INVALID;
  c->link_off.assign((size_t)c->nc + 1, 0);
  for (uint32_t i = 0; i < n_links; ++i) ++c->link_off[src[i] + 1];
  for (uint32_t q = 0; q < c->nc; ++q) c->link_off[q + 1] += c->link_off[q];
  c->link_dst.assign(n_links, 0);
  std::vector<uint32_t> fill(c->link_off.begin(), c->link_off.end() - 1);
  for (uint32_t i = 0; i < n_links; ++i) c->link_dst[fill[src[i]]++] = dst[i];
  return RTM_OK;
}

// Sink strongly-connected components of the links among the flagged set (iterative Tarjan).
rtm_status rtm_hang_roots(rtm_ctx *c, uint32_t window, uint32_t *comp_ids, uint32_t cap, uint32_t *n_roots) {
  if (!c || !n_roots || (cap && !comp_ids)) return RTM_E_INVALID;
  if (c->sticky) return (rtm_status)c->sticky;
  if (!c->have) return RTM_E_STATE;
  if (window >= c->W) return RTM_E_INVALID;
  if (!c->tables_synced) {
    if (c->sum[window].n_hung == 0) {
      *n_roots = 0;
      return RTM_OK;
    }
    return RTM_E_STATE;
  }
  std::vector<uint32_t> F;
  rtm_status s = hung_list(c, window, F);
  if (s) return s;
  const size_t m = F.size();
  auto local = [&](uint32_t comp) -> int64_t {  // index in F (sorted) or -1
    auto it = std::lower_bound(F.begin(), F.end(), comp);
    return (it != F.end() && *it == comp) ? (int64_t)(it - F.begin()) : -1;
  };
  std::vector<std::vector<uint32_t>> adj(m);  // links restricted to flagged components
  if (!c->link_off.empty())
    for (size_t i = 0; i < m; ++i)
      for (uint32_t e = c->link_off[F[i]]; e < c->link_off[F[i] + 1]; ++e) {
        const int64_t j = local(c->link_dst[e]);
        if (j >= 0) adj[i].push_back((uint32_t)j);
      }
  const uint32_t kNone = 0xFFFFFFFFu;
  std::vector<uint32_t> idx(m, kNone), low(m, 0), comp(m, kNone), stk;
  std::vector<uint8_t> on(m, 0);
  uint32_t counter = 0, n_scc = 0;
  std::vector<std::pair<uint32_t, uint32_t>> call;  // (node, next edge)
  for (size_t r = 0; r < m; ++r) {
    if (idx[r] != kNone) continue;
    call.push_back({(uint32_t)r, 0});
    while (!call.empty()) {
      const uint32_t v = call.back().first;
      uint32_t &ei = call.back().second;
      if (ei == 0 && idx[v] == kNone) {
        idx[v] = low[v] = counter++;
        stk.push_back(v);
        on[v] = 1;
      }
      if (ei < adj[v].size()) {
        const uint32_t w = adj[v][ei++];
        if (idx[w] == kNone) call.push_back({w, 0});
        else if (on[w]) low[v] = std::min(low[v], idx[w]);
        continue;
      }
      if (low[v] == idx[v]) {  // v roots an SCC
        uint32_t x;
        do {
          x = stk.back();
          stk.pop_back();
          on[x] = 0;
          comp[x] = n_scc;
        } while (x != v);
        ++n_scc;
      }
      call.pop_back();
      if (!call.empty()) {
        const uint32_t u = call.back().first;
        low[u] = std::min(low[u], low[v]);
      }
    }
  }
  std::vector<uint8_t> sink(n_scc, 1);  // an SCC with a link to another SCC is not a sink
  for (size_t i = 0; i < m; ++i)
    for (uint32_t j : adj[i])
      if (comp[j] != comp[i]) sink[comp[i]] = 0;
  uint32_t n = 0;
  for (size_t i = 0; i < m; ++i)
    if (sink[comp[i]]) {
      if (n < cap) comp_ids[n] = F[i];
      ++n;
    }
  *n_roots = n;
  return RTM_OK;
}

rtm_status rtm_buffer_stats(rtm_ctx *c, uint32_t first, uint32_t count, rtm_buffer_stat *out) {
  if (!c || (count && !out)) return RTM_E_INVALID;
  if (c->sticky) return (rtm_status)c->sticky;
  if (!c->have) return RTM_E_STATE;
  const bool by_gid = c->gid.p != nullptr;
  if ((uint64_t)first + count > (by_gid ? c->n_global : c->nb)) return RTM_E_INVALID;
  if (!c->tables_synced) return RTM_E_STATE;  // world > 1: rtm_sync_tables first
  if (!count) return RTM_OK;
  CK(cudaSetDevice(c->device));
  CK(cudaMemcpyAsync(out, (rtm_buffer_stat *)(by_gid ? c->bstat_g.p : c->bstat.p) + first,
                     (size_t)count * sizeof(rtm_buffer_stat),
                     cudaMemcpyDeviceToHost, c->st));
  CK(cudaStreamSynchronize(c->st));
  for (uint32_t i = 0; i < count; ++i) out[i].reserved = 0;
  return RTM_OK;
}

rtm_status rtm_use_graphs(rtm_ctx *c, int32_t mode) {
  if (!c || mode < RTM_GRAPHS_OFF || mode > RTM_GRAPHS_ALWAYS) return RTM_E_INVALID;
  c->graph_mode = mode;
  if (mode == RTM_GRAPHS_OFF) graphs_clear(c);
  return RTM_OK;
}

rtm_status rtm_graph_stats(rtm_ctx *c, uint64_t *captured, uint64_t *replayed) {
  if (!c || !captured || !replayed) return RTM_E_INVALID;
  *captured = c->graph_captures;
  *replayed = c->graph_replays;
  return RTM_OK;
}

rtm_status rtm_profile(rtm_ctx *c, int32_t enable) {
  if (!c) return RTM_E_INVALID;
  c->prof = enable != 0;
  for (int i = 0; i < KT_N; ++i) {
    c->timers[i] = KernelTimer();
    c->timers[i].name = kKernelNames[i];
  }
  c->marks.clear();
  c->ev_next = 0;
  return RTM_OK;
}

rtm_status rtm_profile_read(rtm_ctx *c, rtm_kernel_time *out, uint32_t cap, uint32_t *n) {
  if (!c || !n || (cap && !out)) return RTM_E_INVALID;
  uint32_t m = 0;
  for (int i = 0; i < KT_N; ++i) {
    if (m < cap) {
      out[m].name = kKernelNames[i];
      out[m].launches = c->timers[i].launches;
      out[m].total_ms = c->timers[i].total_ms;
      out[m].algo_bytes = c->timers[i].algo_bytes;
    }
    ++m;
  }
  *n = m;
  return RTM_OK;
}

}  // extern "C"
