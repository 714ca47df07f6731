/*
 * include/rtm.h — C ABI of the B200 monitoring-snapshot reducer (librtm.so).
 *
 * The reducer turns a stream of simulator trace records into the state a real-time
 * monitor such as AkitaRTM shows (Mosallaei, Isaacs, Sun, "Looking into the Black Box:
 * Monitoring Computer Architecture Simulations in Real-Time with AkitaRTM"; PAPER.md):
 *   - the Bottleneck Analyzer buffer list: a snapshot of all buffers sorted by fullness
 *     percentage or by number of elements (Fig. 3);
 *   - buffer fullness over time: per buffer last / max / min level and the int64
 *     time-weighted occupancy integral (L175-L181, L199);
 *   - progress bars with finished / executing / not-started task counts (L91, L131);
 *   - a hang flag for components whose buffers stay full while their task counts stop
 *     changing (T3 L67-L71; case study 2 L227-L229).
 * The paper gives no formula; the exact definition this library computes is DESIGN.md §2
 * and every reading where the paper is silent is listed in DESIGN.md §3.  All integer
 * outputs are bit-exact with the CPU oracle (oracle/); mean occupancy is one IEEE division.
 *
 * Conventions
 *   - Every call returns rtm_status.  RTM_E_INVALID leaves all state unchanged.
 *     RTM_E_ORDER / RTM_E_CUDA / RTM_E_STATE are sticky: every later call on the context
 *     returns the same code until rtm_reset() or rtm_destroy().
 *   - A context is bound to one CUDA device and one stream and is NOT thread-safe.
 *   - Invalid records are not errors: they are dropped and counted (rtm_window_summary).
 *   - The caller owns every array passed in or out.  Configuration tables are copied at
 *     rtm_create.  Host output pointers must hold the documented number of elements.
 *   - Memory: all device buffers are allocated with cudaMalloc on cfg->device at create
 *     (registry, per-buffer / per-component state) or on first use and grown
 *     (per-call workspaces); nothing is freed before rtm_destroy.
 */
#ifndef RTM_H
#define RTM_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct rtm_ctx rtm_ctx; /* opaque, owned by the library */

typedef enum {
  RTM_OK = 0,
  RTM_E_INVALID = -1,   /* bad argument; no state change                                  */
  RTM_E_CUDA = -2,      /* CUDA runtime failure (sticky)                                  */
  RTM_E_COMM = -3,      /* cross-rank exchange callback failed (sticky)                   */
  RTM_E_ORDER = -4,     /* field-valid records not non-decreasing in ts (sticky)           */
  RTM_E_TOO_SMALL = -5, /* output capacity too small (no state change)                    */
  RTM_E_STATE = -6,     /* call not valid in the current state (e.g. no reduce yet)        */
  RTM_E_NOMEM = -7      /* device allocation failed (sticky)                              */
} rtm_status;

enum { RTM_MEM_HOST = 0, RTM_MEM_DEVICE = 1 };
/* Which buffers count toward the hang condition (a component with such a buffer for the whole
 * window and no task event, H windows in a row, is flagged):
 * RTM_HANG_FULL: a buffer at capacity the whole window (R9, the default);
 * RTM_HANG_NONEMPTY: a buffer non-empty the whole window — the paper's own, looser sign: "if
 *   there is any content in a buffer, we know the buffer owner cannot proceed" (L229; SURVEY.md
 *   §8(f) row 4).  It also flags components backed up behind the stuck one (back-pressure,
 *   L229); rtm_hang_roots separates those given the component connection graph. */
enum { RTM_HANG_FULL = 0, RTM_HANG_NONEMPTY = 1 };
/* "sort the buffers by their fullness percentage or by the number of elements" */
enum { RTM_RANK_PERCENT = 0, RTM_RANK_SIZE = 1,
       /* persistence ranking (a buffer "repeatedly at the top of the list"
        * is the bottleneck, L173, L197-L199): the window's time-weighted mean occupancy
        * integral / (capacity * window length), descending, ties by buffer_id.  Every window of a
        * call must be shorter than 2^32 ticks (else RTM_E_INVALID).  world > 1: each rank ranks its
        * owned buffers and the exchange pack carries the 64-bit order key of every candidate, so
        * the merge ranks the union exactly. */
       RTM_RANK_MEAN = 2 };

/* ---- trace records (16 B each, little-endian, naturally aligned) --------------------------
 * rtm_level_sample: buffer `buffer_id` holds `level` elements of `capacity` from tick ts on
 *   (the "Size" and "Cap" columns of Fig. 3; ts is an integer simulation tick).
 * rtm_task_event: START or END of one task (e.g. a thread block of a GPU kernel, L91, L131).
 *   meta = component_id (bits 0..19) | kernel_id (bits 20..30) | kind (bit 31: 0 START, 1 END)
 * Field-valid sample: buffer_id < n_buffers, capacity == registered capacity, level <= capacity.
 * Field-valid event:  component_id < n_components, kernel_id < n_kernels, bar kernel_id live
 *   (rtm_bar_destroy frees an id; every registered bar starts live).
 * Ordering contract: within the records pending at one rtm_window_reduce call, the ts of
 * field-valid samples is non-decreasing in ingest order, and likewise for field-valid events
 * (reading R15).  A violation makes the call fail with RTM_E_ORDER (sticky).       */
typedef struct {
  int64_t ts;
  uint32_t buffer_id;
  uint16_t level;
  uint16_t capacity;
} rtm_level_sample;

typedef struct {
  int64_t ts;
  uint32_t task_id;
  uint32_t meta;
} rtm_task_event;

#define RTM_META(comp, kernel, kind) \
  (((uint32_t)(comp) & 0xFFFFFu) | (((uint32_t)(kernel) & 0x7FFu) << 20) | ((uint32_t)(kind) << 31))

/* Cross-rank exchange hook (world > 1): gather `bytes` from every rank's device buffer `send`
 * into `recv` (world * bytes, rank-major) on the context's device; must be complete when it
 * returns (the library synchronises its stream before calling).  Returns 0 on success.
 * The Python binding implements it with torch.distributed.all_gather_into_tensor (NCCL). */
typedef int (*rtm_allgather_fn)(void *user, const void *send, void *recv, uint64_t bytes);

/* ---- configuration (≈ RegisterComponent + CreateProgressBar) ------------------ */
typedef struct {
  uint32_t n_buffers;               /* 1 .. 2^20 (1048576; larger: RTM_E_INVALID)              */
  uint32_t n_components;            /* 1 .. 2^20                                               */
  uint32_t n_kernels;               /* progress bars, 1 .. 2048                                */
  const uint32_t *buffer_owner;     /* host [n_buffers]: owning component id                   */
  const uint16_t *buffer_capacity;  /* host [n_buffers]: 1 .. 65534 (65535 is reserved)        */
  const int64_t *kernel_total;      /* host [n_kernels]: planned tasks per bar                 */
  int64_t t0;                       /* begin of the first window                               */
  uint32_t hang_windows;            /* H >= 1: consecutive windows before a hang is flagged    */
  uint32_t k;                       /* top-k computed for every window, 1 .. 1024              */
  int32_t rank_mode;                /* RTM_RANK_PERCENT, RTM_RANK_SIZE or RTM_RANK_MEAN        */
  int32_t device;                   /* CUDA device ordinal                                     */
  int32_t rank, world;              /* world == 1: single GPU; else this context is one shard;
                                       world * k <= 8192 (merge candidates in shared memory)   */
  const uint8_t *owned_components;  /* host [n_components] or NULL (= all): components whose
                                       buffers and events this rank holds (ranking restricted) */
  rtm_allgather_fn allgather;       /* required when world > 1                                 */
  void *allgather_user;
  void *stream;                     /* cudaStream_t to run on (NULL = the legacy default)      */
  /* Rank-local buffer numbering (owner sharding without a global registry on every rank):
   * when buffer_global_id is set, this context registers only its own buffers as a dense local
   * numbering 0..n_buffers-1, records carry LOCAL buffer ids, and every result reports GLOBAL
   * ids: top-k entries, the digest's buffer id, and the per-buffer table (indexed by global id,
   * n_global_buffers entries).  Global ids must be strictly increasing in the local id, so ties
   * broken by local id agree with ties by global id.  pack_buffers (world > 1) = the largest
   * n_buffers over the ranks (equal-size exchange packs); 0 means n_buffers.                   */
  const uint32_t *buffer_global_id; /* host [n_buffers] or NULL (ids are global)               */
  uint32_t n_global_buffers;        /* > every global id; 0 when buffer_global_id is NULL       */
  uint32_t pack_buffers;
  int32_t hang_mode;                /* RTM_HANG_FULL (0, default) or RTM_HANG_NONEMPTY          */
  int32_t allgather_on_stream;      /* world > 1: nonzero = `allgather` enqueues the collective on
                                       `stream` (e.g. NCCL) and may return before it completes; the
                                       library then never synchronises the host around it      */
} rtm_config;

/* ---- per-window outputs --------------------------------------------------------------------- */
typedef struct {
  int64_t t_begin, t_end;           /* window [t_begin, t_end)                                 */
  uint64_t n_samples, n_events;     /* kept records                                            */
  uint64_t n_dropped;               /* dropped samples + events charged to this window         */
  uint64_t digest;                  /* sum over touched buffers of the DESIGN.md §2 mixer      */
  uint32_t n_touched, n_hung;       /* buffers with >= 1 kept sample; flagged components       */
} rtm_window_summary;               /* 56 B */

typedef struct { uint32_t buffer_id; uint16_t level, capacity; } rtm_topk_entry; /* Fig. 3 row */
typedef struct { int64_t total, started, finished, in_flight, not_started; } rtm_progress_entry;
typedef struct { int64_t started, finished, in_flight; } rtm_component_tasks;
typedef struct {
  int64_t integral;                 /* sum level*dt over the window (mod 2^64)                  */
  uint16_t last, max, min, capacity;
  uint32_t n_samples, reserved;
  double mean_occ;                  /* (double)integral / (double)(capacity * (t_end-t_begin)) */
} rtm_buffer_stat;                  /* 32 B */

typedef struct {
  const char *name;                 /* kernel name                                              */
  uint32_t launches;                /* launches timed since rtm_profile(ctx, 1)                 */
  double total_ms;                  /* summed CUDA-event durations on the context's stream      */
  uint64_t algo_bytes;              /* algorithmic bytes those launches had to move             */
} rtm_kernel_time;

/* ---- API -------------------------------------------------------------------------------------- */
/* Validate cfg, copy the registry to the device, allocate state (levels start at 0: buffers
 * start empty, L229).  *out receives the context.  RTM_E_INVALID for out-of-range fields. */
rtm_status rtm_create(const rtm_config *cfg, rtm_ctx **out);
void rtm_destroy(rtm_ctx *ctx);
/* Back to the state right after rtm_create (t_prev = t0, levels 0, counters 0, no error). */
rtm_status rtm_reset(rtm_ctx *ctx);

/* Append records to the pending stream of the next rtm_window_reduce (ingest order = call
 * order, then array order).  mem = RTM_MEM_HOST: copied host->device now (pinned memory is
 * copied asynchronously on the context stream).  mem = RTM_MEM_DEVICE: pointers on the
 * context's device; a single device ingest is zero-copy and must stay valid until the next
 * rtm_window_reduce returns; further device ingests are copied into an internal buffer.
 * Either pointer may be NULL when its count is 0. */
rtm_status rtm_ingest(rtm_ctx *ctx, const rtm_level_sample *samples, uint64_t n_samples,
                      const rtm_task_event *events, uint64_t n_events, int32_t mem);

/* THE HOT PATH.  Reduce all pending records over n_windows consecutive windows
 * [t_prev, t_end[0]), [t_end[0], t_end[1]), ... (t_end host array, non-decreasing,
 * t_end[0] >= t_prev, each window shorter than 2^40 ticks, else RTM_E_INVALID with no state
 * change).  Records outside
 * [t_prev, t_end[n-1]) are dropped and counted, not carried.  Blocks until the per-window
 * summaries, top-k lists and progress bars are on the host; `out` (host, nullable)
 * receives n_windows summaries.  With world > 1 every rank must call it with the same
 * t_end (collective); all ranks then return identical merged results. */
rtm_status rtm_window_reduce(rtm_ctx *ctx, const int64_t *t_end, uint32_t n_windows, rtm_window_summary *out);

/* Results of the most recent rtm_window_reduce; `window` indexes its batch.
 * world > 1: the per-window results above (summaries, top-k, progress bars) are merged by every
 * reduce.  The per-buffer table, the per-component totals and the hang lists are exchanged only
 * on demand (rtm_sync_tables, or rtm_tables_local + rtm_tables_merge): until then
 * rtm_buffer_stats, rtm_progress with comps, and rtm_hang_check / rtm_hang_roots of a window
 * whose merged n_hung is nonzero return RTM_E_STATE (windows with n_hung == 0 answer empty). */
/* Bottleneck Analyzer list (L173): min(k, eligible buffers) entries, most occupied first,
 * ties by buffer_id ascending.  out holds k entries. */
rtm_status rtm_topk_buffers(rtm_ctx *ctx, uint32_t window, rtm_topk_entry *out, uint32_t *n_out);
/* Progress bars after `window` (L131): bars[n_kernels].  comps[n_components] (nullable) is
 * only available for the last window of the batch (else RTM_E_INVALID). */
rtm_status rtm_progress(rtm_ctx *ctx, uint32_t window, rtm_progress_entry *bars, rtm_component_tasks *comps);
/* Hang-flagged component ids of `window`, ascending.  Writes min(cap, n) ids; *n_hung = n. */
rtm_status rtm_hang_check(rtm_ctx *ctx, uint32_t window, uint32_t *comp_ids, uint32_t cap, uint32_t *n_hung);
/* Hang root causes (L229-L235, L342-L344).  The paper finds the stuck
 * components by hand: flagged components may only be backed up behind the real culprit
 * ("caused by buffer backpressure", L229; "L1 cache and DRAM controllers cannot make progress
 * because they cannot send messages to L2 caches", L235) and names a graph of component
 * connections as the missing view (L342-L344).  Given that graph:
 * rtm_set_links: n_links directed links, component src[i] sends to component dst[i] (host
 *   arrays; replaces the previous graph; ids < n_components, else RTM_E_INVALID).
 * rtm_hang_roots: among the components flagged in `window` (last batch), the members of the
 *   sink strongly-connected components of the links restricted to flagged components: a
 *   circular wait (case study 2, L217) or a stuck component whose successors are not flagged;
 *   components flagged only because they wait on one of those are left out.  Ascending ids;
 *   writes min(cap, n) ids, *n_roots = n.  Computed on the host from the window's flagged set. */
rtm_status rtm_set_links(rtm_ctx *ctx, const uint32_t *src, const uint32_t *dst, uint32_t n_links);
rtm_status rtm_hang_roots(rtm_ctx *ctx, uint32_t window, uint32_t *comp_ids, uint32_t cap, uint32_t *n_roots);
/* Full per-buffer table of the last window of the batch for buffers [first, first+count)
 * (global ids when the context uses a rank-local numbering; buffers of no rank read as zero). */
rtm_status rtm_buffer_stats(rtm_ctx *ctx, uint32_t first, uint32_t count, rtm_buffer_stat *out);

/* Bulk form of the three accessors above for windows [first, first+count) of the last batch:
 * topk[count*k] + topk_n[count], bars[count*n_kernels], summaries[count]; each nullable. */
rtm_status rtm_window_results(rtm_ctx *ctx, uint32_t first, uint32_t count, rtm_window_summary *summaries,
                              rtm_topk_entry *topk, uint32_t *topk_n, rtm_progress_entry *bars);

/* Two-phase form of rtm_window_reduce for callers that run the exchange themselves:
 * reduce_local computes this rank's results and packs them; *pack / *pack_bytes give the
 * device buffer to all-gather; rtm_merge consumes world*pack_bytes gathered bytes (device).
 * The pack is owned by the context and valid until its next reduce call, and complete in the
 * context stream's order (consume it on that stream, or synchronise first); its size depends on
 * n_windows, k, the pack size in buffers and the rank mode (MEAN adds each candidate's 64-bit
 * order key), so every rank must use the same configuration.  Between a successful
 * reduce_local and its rtm_merge the context is merge-pending: another reduce (local or not)
 * and rtm_watch return RTM_E_STATE (no state change); rtm_reset clears the pending merge and
 * the call's effects.  Errors: RTM_E_INVALID (null arguments), RTM_E_STATE (rtm_merge without
 * a preceding reduce_local, or a second reduce while merge-pending), the reduce's own. */
rtm_status rtm_window_reduce_local(rtm_ctx *ctx, const int64_t *t_end, uint32_t n_windows,
                                   const void **pack, uint64_t *pack_bytes);
rtm_status rtm_merge(rtm_ctx *ctx, const void *gathered, uint32_t world, rtm_window_summary *out);

/* Bytes of the per-call exchange pack (world > 1): kWinFields x 8 + k x 8 (+ k x 8 in rank mode
 * MEAN) + 4 + n_kernels x 8 per window; a pure function, no context. */
uint64_t rtm_exchange_bytes(uint32_t n_windows, uint32_t k, uint32_t n_kernels, int32_t rank_mode);

/* On-demand exchange of the last call's tables (world > 1, collective: every rank calls it
 * after the same reduce).  rtm_sync_tables runs it through the config's allgather callback;
 * rtm_tables_local / rtm_tables_merge are its two-phase form: *pack (device, owned by the
 * context, complete in the context stream's order) holds this rank's per-component totals,
 * per-buffer table of the last window and per-window hang bitmaps; rtm_tables_merge consumes
 * world * bytes gathered bytes (device, rank-major).  RTM_E_STATE before the first reduce. */
rtm_status rtm_sync_tables(rtm_ctx *ctx);
rtm_status rtm_tables_local(rtm_ctx *ctx, const void **pack, uint64_t *bytes);
rtm_status rtm_tables_merge(rtm_ctx *ctx, const void *gathered, uint32_t world);

/* ---- Progress bar registry (CreateProgressBar / UpdateProgressBar / DestroyProgressBar, PAPER.md
 * L99; progress bars L131).  Bar ids are the kernel_id field of task
 * events, 0 <= id < n_kernels; every bar registered at rtm_create starts live.  Calls take
 * effect at the next rtm_window_reduce (stream-ordered); with world > 1 every rank must make the
 * same calls.
 * rtm_bar_create: the lowest free id becomes live with `total` tasks and zero counts; *bar_id
 *   receives it.  RTM_E_TOO_SMALL (no state change) when all n_kernels ids are live.
 * rtm_bar_update: set a live bar's total (not_started = total - started).
 * rtm_bar_destroy: free a live id.  Task events naming a free id are field-invalid (dropped and
 *   counted) until it is created again; its progress entry reads all zero.
 * RTM_E_INVALID (no state change) for an id that is out of range or not live. */
rtm_status rtm_bar_create(rtm_ctx *ctx, int64_t total, uint32_t *bar_id);
rtm_status rtm_bar_update(rtm_ctx *ctx, uint32_t bar_id, int64_t total);
rtm_status rtm_bar_destroy(rtm_ctx *ctx, uint32_t bar_id);

/* Windows-in-top-k counter (persistence): for buffers [first,
 * first+count) (global ids with a rank-local numbering), the number of windows since create /
 * reset in which the buffer was in the window's top-k list (the merged list when world > 1).
 * out (host) holds count entries. */
rtm_status rtm_topk_persistence(rtm_ctx *ctx, uint32_t first, uint32_t count, uint32_t *out);

/* ---- Value monitor (§IV-C.3, Fig. 2 F) ----------
 * The dashboard plots "up to five values" over time and keeps "the last 300 data points"
 * (L175, L179).  Here a watched buffer's value per window is its rtm_buffer_stat of that window
 * (last / max / min level, integral, mean occupancy): every window of every reduce appends one
 * point per watched buffer to that buffer's ring of the last RTM_WATCH_POINTS windows.  The
 * points are produced by the fold kernel in the same pass as the snapshot (no extra pass over
 * the records) and copied back with the call's results.  With world > 1 a ring fills on the
 * rank that owns the buffer; the other ranks' rings for it stay empty. */
enum { RTM_WATCH_MAX = 5, RTM_WATCH_POINTS = 300 };
typedef struct {
  int64_t t_end;                    /* end of the window the point describes                  */
  rtm_buffer_stat stat;             /* that window's statistics of the watched buffer         */
} rtm_watch_point;                  /* 40 B */
/* Replace the watched set by buffer_ids[0..n) (n <= RTM_WATCH_MAX, distinct, < n_buffers;
 * global ids with a rank-local numbering) and clear every ring; n = 0 stops watching.
 * RTM_E_INVALID (no state change) for n > RTM_WATCH_MAX, duplicates or out-of-range ids;
 * RTM_E_STATE while a merge is pending (rtm_window_reduce_local without rtm_merge). */
rtm_status rtm_watch(rtm_ctx *ctx, const uint32_t *buffer_ids, uint32_t n);
/* The ring of watched slot `slot` (order given to rtm_watch), oldest point first:
 * out[RTM_WATCH_POINTS] (host) receives min(points so far, RTM_WATCH_POINTS) points,
 * *n_out that count.  RTM_E_INVALID for slot >= the watched count. */
rtm_status rtm_watch_series(rtm_ctx *ctx, uint32_t slot, rtm_watch_point *out, uint32_t *n_out);

/* Launch mechanism of rtm_window_reduce / rtm_window_reduce_local (results are identical).
 * The call's kernels and copies form a fixed sequence for a given launch shape (window count,
 * tile counts of the pending records, partition / fold variant): it can be captured once into a
 * CUDA graph and replayed with only the kernels' arguments replaced, which removes the per-kernel
 * launch cost of small calls (the list is refreshed for every window).
 *   RTM_GRAPHS_OFF     direct launches
 *   RTM_GRAPHS_AUTO    graphs for calls of <= 64 windows (default)
 *   RTM_GRAPHS_ALWAYS  graphs for every call
 * Up to 8 shapes are cached per context (least recently used evicted); a workspace growth drops
 * them.  Profiling (rtm_profile) uses direct launches.  If the driver cannot capture the sequence
 * the context falls back to direct launches for good.  RTM_E_INVALID for another mode. */
typedef enum { RTM_GRAPHS_OFF = 0, RTM_GRAPHS_AUTO = 1, RTM_GRAPHS_ALWAYS = 2 } rtm_graph_mode;
rtm_status rtm_use_graphs(rtm_ctx *ctx, int32_t mode);
/* Calls of this context launched from a newly captured graph / by replaying a cached one
 * (host outputs; the rest were direct launches). */
rtm_status rtm_graph_stats(rtm_ctx *ctx, uint64_t *captured, uint64_t *replayed);

/* Per-kernel CUDA-event timing on the context stream (off by default). */
rtm_status rtm_profile(rtm_ctx *ctx, int32_t enable);
rtm_status rtm_profile_read(rtm_ctx *ctx, rtm_kernel_time *out, uint32_t cap, uint32_t *n);

const char *rtm_status_str(rtm_status s);
/* Build identification string ("librtm sm_100a ..."). */
const char *rtm_version(void);
/* Kernel launches issued by this library in this process so far (all contexts, all streams).
 * Monotone; callers take differences around a region to count the kernels it launched. */
uint64_t rtm_kernel_launches(void);

#ifdef __cplusplus
}
#endif
#endif /* RTM_H */
