/*
 * oracle/oracle.h — plain, slow, obviously-correct CPU oracle for the monitoring-snapshot
 * reduction (TEST INFRASTRUCTURE ONLY).
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference leg
 * may load liboracle.so.  It shares no code, header, table or helper with the CUDA path
 * (paper_conf_micro_mosallaeii024_b200/): the record structs below are re-declared from
 * the specification text, not included from include/rtm.h.
 *
 * What it computes is the definition in DESIGN.md §2, written out
 * window by window in the paper's vocabulary:
 *   - buffer snapshot: per buffer last / max / min level and the time-weighted occupancy
 *     integral  I = sum level * dt  ("snapshot of all the buffers",
 *     L181/L199 "fullness of a buffer ... over time");
 *   - Bottleneck Analyzer list: all buffers sorted by fullness percentage or by number of
 *     elements, most occupied first (L137-L157 Fig. 3);
 *   - progress bars: finished / executing / not started task counts (L91, L131);
 *   - hang flag: components whose buffers stay full while their task counts stop
 *     changing (L67-L71 T3, L227-L229 case study 2).
 * The paper fixes none of the formulas; every reading taken is listed in DESIGN.md §3.
 */
#ifndef RTM_ORACLE_H
#define RTM_ORACLE_H
#include <stdint.h>

typedef struct { int64_t ts; uint32_t buffer_id; uint16_t level; uint16_t capacity; } orc_sample;
typedef struct { int64_t ts; uint32_t task_id; uint32_t meta; } orc_event;

typedef struct {
  uint32_t n_buffers, n_components, n_kernels;
  const uint32_t *buffer_owner;    /* [n_buffers] */
  const uint16_t *buffer_capacity; /* [n_buffers], >= 1 */
  const int64_t *kernel_total;     /* [n_kernels] */
  int64_t t0;
  uint32_t hang_windows;           /* H >= 1 */
  uint32_t k;
  int32_t rank_mode;               /* 0 percent, 1 size, 2 window mean occupancy */
  const uint8_t *owned;            /* [n_components] nullable: shard ownership, restricts ranking */
  int32_t hang_mode;               /* 0: a buffer full all window; 1: non-empty all window (L229) */
} orc_config;

typedef struct {
  int64_t t_begin, t_end;
  uint64_t n_samples, n_events, n_dropped, digest;
  uint32_t n_touched, n_hung;
} orc_summary;

typedef struct { uint32_t buffer_id; uint16_t level, capacity; } orc_topk;
typedef struct { int64_t total, started, finished, in_flight, not_started; } orc_progress;
typedef struct {
  int64_t integral;
  uint16_t last, max, min, capacity;
  uint32_t n_samples, pad;
  double mean_occ;
} orc_bstat;
typedef struct { int64_t started, finished, in_flight; } orc_comp;

typedef struct orc_ctx orc_ctx;

orc_ctx *orc_create(const orc_config *cfg);
void orc_persistence(const orc_ctx *c, uint32_t *out); /* [n_buffers] windows in the top-k */
int orc_bar_create(orc_ctx *c, int64_t total, uint32_t *id);
int orc_bar_update(orc_ctx *c, uint32_t id, int64_t total);
int orc_bar_destroy(orc_ctx *c, uint32_t id);
void orc_destroy(orc_ctx *c);
void orc_reset(orc_ctx *c);

/* Reduce the given pending records over windows [t_prev, t_end[0]), [t_end[0], t_end[1]), ...
 * Outputs (nullable unless stated): sum[W] (required), topk[W*k] + topk_n[W], prog[W*n_kernels],
 * hung[W*n_components] (0/1 flags), last_stats[n_buffers] (latest window), comps[n_components]
 * (latest window), all_stats[W*n_buffers] (every window's full per-buffer table).
 * Returns 0, -1 (invalid arguments, no state change), -4 (ts order violated, sticky). */
int orc_reduce(orc_ctx *c, const orc_sample *s, uint64_t ns, const orc_event *e, uint64_t ne,
               const int64_t *t_end, uint32_t W, orc_summary *sum, orc_topk *topk, uint32_t *topk_n,
               orc_progress *prog, uint8_t *hung, orc_bstat *last_stats, orc_comp *comps,
               orc_bstat *all_stats);

/* The digest mixer of DESIGN.md §2 (exposed for pinning). */
uint64_t orc_digest_term(uint32_t b, uint16_t last, uint16_t mx, uint16_t mn, uint16_t cap, uint32_t n,
                         int64_t integral);

/* Multi-shard merge: merges per-shard window results into whole-trace ones. */
int orc_merge_topk(const orc_topk *const *shard_topk, const uint32_t *const *shard_n, uint32_t n_shards,
                   uint32_t W, uint32_t k, int32_t rank_mode, orc_topk *out, uint32_t *out_n);

#endif
