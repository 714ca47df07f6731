// rtm_internal.h — device data layout and kernel launchers of librtm (sm_100a).
//
// Data path of one rtm_window_reduce call (DESIGN.md §4 has the rationale and rooflines):
//   K0 prep       : one cooperative launch: zero the call's accumulators; per window boundary,
//                   warp 33-ary search for the first record position whose field-valid successors
//                   all have ts >= boundary -> region [B_r, B_r+1) per window; grid sync; region ->
//                   tile tables; grid sync; per-tile descriptors
//   K1 partition  : one CTA per 4096-sample tile of one region; validate, order-check, stable
//                   multisplit of kept samples by 256-buffer bin into 8-byte staging entries
//   K1b subpart   : (> 170 bins) K1 keys by superbin; per (window, superbin) a stable counting sort
//                   by bin into (window, bin)-contiguous staging
//   K3 events     : one CTA per 4096-event tile; progress deltas, component activity bitmaps
//   K2 fold       : one warp per (window, bin) unit, dequeued in window order; in-order fold of
//                   the bin's samples (delta form of the integral), carry-in resolved by
//                   decoupled look-back over earlier windows' last levels, finalize + digest
//   K4 order check: cross-tile ts monotonicity of field-valid records
//   K5 top-k      : one CTA per window, MSB radix select on the exact 32-bit fullness key
//   K6 hang       : per component run length over windows
//   K7 progress   : per kernel prefix over windows, component totals
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include <string>
#include <vector>

#include "rtm.h"

namespace rtm {

constexpr int kBin = 256;                   // buffers per bin (bin_log 8); bin_log 9: 512
constexpr int kTileS = 4096;                // samples per partition tile
constexpr int kTileE = 4096;                // events per event tile
constexpr int kK1Threads = 256;             // 8 warps x 512-sample sub-tiles
constexpr int kK3Threads = 256;
#ifndef RTM_FOLD_WARPS
#define RTM_FOLD_WARPS 4
#endif
constexpr int kFoldWarps = RTM_FOLD_WARPS;  // warps per fold CTA (compile-time A/B override)
constexpr uint16_t kSent = 0xFFFFu;         // "no kept sample in this window" marker
constexpr uint32_t kMaxBins = 4096;         // n_buffers <= 2^20 (fallback partition smem 160 KB)
constexpr uint32_t kTopkSmemKeys = 40960;
constexpr uint32_t kTInline = 16;           // window bounds passed inline for W + 1 <= 16
constexpr uint32_t kLmMaxBins = 170;        // lane-major partition: count rows (bins x 48 B) fit a warp's 8 KB slot
constexpr int kSupLog = 14;                 // two-pass partition: superbins of 2^14 buffers (<= 64 of them)   // keys held in shared memory by the top-k kernel
// ts offset field of a staging entry: 48 - bin_log bits (entry = off << (16 + bin_log) | level << bin_log | lid)
inline int64_t max_window_len(int bin_log) { return (int64_t)1 << (bin_log >= 8 ? 40 : 48 - bin_log > 40 ? 40 : 48 - bin_log); }

// per-window scalar accumulators, SoA [kWinFields][W] u64
enum { WF_SAMPLES = 0, WF_EVENTS, WF_DROPPED, WF_DIGEST, WF_TOUCHED, WF_HUNG, kWinFields };

struct TileDesc {            // per sample tile, precomputed so the partition reads one 48-byte record
  long long start;           // first record (index into the sample stream)
  long long lo;              // region lower bound: field-valid records need (u64)(ts - lo) < wlen
  unsigned long long wlen;
  int n;                     // records in the tile
  int window;                // -1: head / tail region
  unsigned charge;           // window the tile's drops are charged to
  unsigned pad[3];
};
static_assert(sizeof(TileDesc) == 48, "TileDesc is three 16-byte chunks");

struct TileMeta {            // per tile, for the cross-tile order check
  long long first_ts;
  long long last_ts;
  unsigned flags;            // bit0 has valid record, bit1 in-tile order / range violation
  unsigned pad;
};

struct KernelTimer {
  const char *name;
  uint32_t launches = 0;
  double total_ms = 0;
  uint64_t algo_bytes = 0;
};

// Everything a launch needs, by value (kernel parameter).
struct Params {
  // registry
  uint32_t nb, nc, nk, nbins, ncw, k;
  int32_t bin_log;           // buffers per bin = 2^bin_log (8, or 7 for large registries)
  int32_t rank_mode;
  uint32_t H;
  int32_t hang_mode;         // RTM_HANG_FULL / RTM_HANG_NONEMPTY
  const uint16_t *cap;
  const uint32_t *owner;
  const uint8_t *elig;       // [nb] 1 if buffer ranks on this rank
  const int64_t *ktotal;
  const uint8_t *klive;      // [nk] progress bar id in use (rtm_bar_create / rtm_bar_destroy)
  int32_t all_live;          // every bar id live: event validity skips the klive lookup
  const unsigned long long *rcp;  // [65536] floor(2^48 / c) (exact fullness key, K5)
  const uint32_t *elig_ids;  // [n_elig] ascending ids of ranked buffers
  const uint32_t *gid;       // [nb] global buffer id (rank-local numbering) or nullptr
  uint32_t n_global;         // global id space (per-buffer table size) when gid is set
  uint32_t pack_nb;          // per-buffer entries in an exchange pack
  uint32_t n_elig;
  // call
  uint32_t W;                // windows in the call
  int32_t narrow;            // every window shorter than 2^32 ticks (32-bit order check)
  int32_t narrow_d;          // max capacity * every window length < 2^32: the fold's D in 32 bits
  uint32_t epoch;
  const long long *T;        // [W+1]: T[0] = t_begin, T[w+1] = t_end[w]
  // few-window calls (W + 1 <= kTInline): the window bounds travel in the kernel arguments and
  // k_prep writes T (no host-to-device copy in the call's launch sequence)
  int32_t t_inline;
  long long Tin[16];
  const rtm_level_sample *s;
  uint64_t ns;
  const rtm_task_event *e;
  uint64_t ne;
  const long long *Bs;       // [W+3] sample region boundaries (positions)
  const long long *Be;
  const uint32_t *rts;       // [W+3] first tile of each sample region; rts[W+2] = total
  const uint32_t *rte;
  const uint32_t *tile_reg_s;// [n_tiles_s] region of each tile
  const uint32_t *tile_reg_e;
  uint32_t n_tiles_s, n_tiles_e;  // upper bounds (grid sizes); device counts are rts/rte[W+2]
  // outputs / workspaces
  TileDesc *tdesc;           // [n_tiles_s]
  uint16_t *soff;            // [n_tiles_s * (nbins+1)] tile-local bin offsets
  unsigned long long *stage; // [n_tiles_s * kTileS]
  TileMeta *smeta, *emeta;
  uint16_t *lastlvl;         // [W * nb]
  uint32_t *flags;           // [W * nbins]
  unsigned long long *win;   // [kWinFields * W]
  uint32_t *kdelta;          // [W * nk * 2]
  unsigned long long *cdelta;// [nc * 2]
  uint32_t *active;          // [W * ncw]
  uint32_t *anyfull;         // [W * ncw]
  uint32_t *hung;            // [W * ncw]
  uint32_t *hsfx;            // [W * ncw] suffix ANDs of the block-parallel long-H hang path, or nullptr
  uint32_t *unit_ctr;        // [0] fold units dequeued, [1] partition tiles, [2] fused event tiles claimed
  int32_t fuse_events;       // the persistent partition also runs the event tiles (K3 in K1)
  uint32_t *status;          // bit0 sample order, bit1 event order
  const uint16_t *carry_in;  // [nb]
  uint16_t *carry_out;       // [nb]
  const uint32_t *run;       // [nc] carried hang run length (in)
  uint32_t *run_out;         // [nc] (out, ping-pong with run)
  long long *kstart, *kend;  // [nk] cumulative
  long long *cstart, *cend;  // [nc] cumulative
  unsigned long long *topk;  // [W * k] packed (id | level<<32 | cap<<48)
  uint32_t *topk_n;          // [W]
  uint32_t tk_slices;        // top-k slices per window (> 1: few windows, K5 runs per id slice)
  uint32_t tk_slice_len;     // buffers per slice (multiple of 8)
  unsigned long long *tk_scratch;  // [W * tk_slices * k] per-slice candidates (key32 << 32 | ~id)
  long long *prog;           // [W * nk * 5]
  rtm_buffer_stat *bstat;    // [nb] last window, local ids
  rtm_buffer_stat *bstat_g;  // [n_global] merged / scattered table by global id (gid set)
  rtm_component_tasks *comps;// [nc]
  unsigned long long *mkey;  // [W * nb] rank mode MEAN: floor(integral * 2^32 / cap) (exact order key)
  const unsigned long long *rcp64;  // [65536] floor(2^64 / c) (c >= 2)
  unsigned long long *tkey;  // [W * k] MEAN, world > 1: order keys of the local top-k (exchange pack)
  uint32_t *persist;         // [id space] windows in the top-k list
  int32_t persist_inline;    // world == 1: the top-k kernels count their own winners (no k_persist)
  uint32_t n_watch;          // value monitor: watched local buffer ids (0xFFFFFFFF: not on this rank)
  uint32_t watch[RTM_WATCH_MAX];
  rtm_buffer_stat *wstat;    // [W * RTM_WATCH_MAX] per-window statistics of the watched buffers
  unsigned long long *dbg;   // phase-timing scratch (RTM_PHASE_TIMING builds only)
  // two-pass path (> 170 bins, narrow windows): pass 1 partitions by superbin (buffer_id >> kSupLog)
  // into stage / soff (rows of nsb + 1); k_subpart re-partitions every (window, superbin) by bin
  // into stage2, (window, bin)-contiguous: bin b of window w is stage2[woff[w][b] .. woff[w][b+1])
  uint32_t nsb;              // superbins (0: one-pass path)
  unsigned long long *stage2;// [n_tiles_s * kTileS]
  uint32_t *woff;            // [W * (nbins + 1)]
  // range-parallel sequential fold (two-pass path, very sparse calls): the call's windows in
  // seq_ranges ranges of seq_range_len, one unit per (bin, range); endkey[r][b] = max over buffer
  // b's kept samples in range r of (staging index + 1) << 16 | level (k_subpart), 0 if none
  uint32_t seq_ranges, seq_range_len;
  unsigned long long *endkey;  // [(seq_ranges - 1) * nb]
};

// launchers (rtm_kernels.cu); all asynchronous on `st`
struct ClearList;
// clear + region boundaries + tile tables, one cooperative launch (p.Bs/Be/rts/rte/tdesc/tile_reg set)
void launch_prep(const Params &p, const ClearList &cl, long long *Bs, long long *Be, int n_sms, cudaStream_t st);
void launch_partition(const Params &p, int n_sms, cudaStream_t st);
void launch_events(const Params &p, cudaStream_t st);
bool partition_fuses_events(uint32_t nbins, uint32_t n_tiles_s, bool two_pass);  // lane-major partition path
bool partition_two_pass(uint32_t nbins, bool narrow);  // > 170 bins: superbins + k_subpart
bool fold_sequential(const Params &p);  // very sparse call: the sequential fold (one warp per bin)
bool hang_block_path(uint32_t W, uint32_t H);  // long H and W >= H: block-parallel van Herk hang passes
void launch_subpart(const Params &p, int n_sms, cudaStream_t st);
void launch_fold(const Params &p, int n_sms, cudaStream_t st);
void launch_order_check(const Params &p, cudaStream_t st);
void launch_topk(const Params &p, cudaStream_t st);
// slices per window for K5 (1 = one CTA per window); sets *slice_len
uint32_t topk_slices(uint32_t nb, uint32_t k, uint32_t W, int n_sms, bool all, uint32_t *slice_len);
void launch_hang(const Params &p, cudaStream_t st);
void launch_progress(const Params &p, cudaStream_t st);
void launch_persist(const Params &p, cudaStream_t st);
// multi-rank exchange
uint64_t pack_bytes(const Params &p);
void launch_pack(const Params &p, void *pack, cudaStream_t st);
void launch_merge(const Params &p, const void *gathered, uint32_t world, long long *gcum, cudaStream_t st);
uint64_t exchange_bytes(uint32_t W, uint32_t k, uint32_t nk, int rank_mode);  // per-call pack size
uint64_t tables_bytes(const Params &p);
void launch_pack_tables(const Params &p, void *pack, cudaStream_t st);
void launch_merge_tables(const Params &p, const void *gathered, uint32_t world, cudaStream_t st);
bool merge_fits(uint32_t world, uint32_t k);  // world * k candidates fit the merge's shared memory
void launch_scatter_bstat(const Params &p, cudaStream_t st);  // gid set, world == 1
unsigned long long kernel_launches();  // kernels launched by this library in this process
void count_launches(unsigned n);       // kernels launched by a CUDA graph replay
void launch_shape(const Params &p, uint64_t key[3]);  // launch-sequence shape (graph cache key)
const void *prep_kernel_fn();          // k_prep (the one kernel with arguments besides Params)

// Device ranges zeroed by ONE kernel launch (replaces per-buffer cudaMemsetAsync calls).
struct ClearList {
  static constexpr int kMax = 12;
  void *ptr[kMax];
  unsigned long long bytes[kMax];
  int n = 0;
  void add(void *p, size_t b) {
    if (p && b && n < kMax) {
      ptr[n] = p;
      bytes[n] = b;
      ++n;
    }
  }
};
void launch_clear(const ClearList &cl, cudaStream_t st);
void configure_kernels_once();  // opt-in shared-memory limits, once per device
void configure_partition_once();  // (rtm_partition.cu) the partition kernels' shared-memory limits
int occupancy(const void *fn, int threads, size_t smem);  // resident blocks per SM (cached)
bool partition_caps_smem(uint32_t nbins, uint32_t nb);  // the lane-major partition keeps cap[] in shared memory
size_t fold_smem_bytes(int bin_log);
size_t partition_smem_bytes(uint32_t nbins, uint32_t nb);
size_t topk_smem_bytes(uint32_t nb);

}  // namespace rtm
