// rtm_kernels.cu — sm_100a kernels of the window-snapshot reduction (see rtm_internal.h and
// DESIGN.md §4).  No tensor cores: nothing here is a dense contraction; the path is bound by
// the one compulsory HBM read of 16 B per trace record.
#include <cuda_runtime.h>
#include <stdint.h>

#include "rtm_internal.h"

namespace rtm {
namespace {

constexpr unsigned kFull = 0xFFFFFFFFu;
constexpr long long kTsMin = (long long)0x8000000000000000ULL;
constexpr long long kTsMax = 0x7FFFFFFFFFFFFFFFLL;

__device__ __forceinline__ unsigned lanemask_lt() {
  unsigned m;
  asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
  return m;
}
__device__ __forceinline__ int4 ld_stream(const void *p) { return __ldcs(reinterpret_cast<const int4 *>(p)); }
__device__ __forceinline__ long long shfl_ll(long long v, int src) {
  return (long long)__shfl_sync(kFull, (unsigned long long)v, src);
}
__device__ __forceinline__ unsigned long long shfl_xor_ull(unsigned long long v, int m) {
  return __shfl_xor_sync(kFull, v, m);
}
__device__ __forceinline__ long long rec_ts(const int4 &v) {
  return (long long)(((unsigned long long)(unsigned)v.y << 32) | (unsigned)v.x);
}
__device__ __forceinline__ unsigned ld_acquire_u32(const unsigned *p) {
  unsigned v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_release_u32(unsigned *p, unsigned v) {
  asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ unsigned short ld_relaxed_u16(const unsigned short *p) {
  unsigned short v;
  asm volatile("ld.relaxed.gpu.global.u16 %0, [%1];" : "=h"(v) : "l"(p) : "memory");
  return v;
}

// field validity (include/rtm.h)
__device__ __forceinline__ bool sample_valid(const Params &p, const int4 &v) {
  unsigned b = (unsigned)v.z, lvl = (unsigned)v.w & 0xFFFFu, c = (unsigned)v.w >> 16;
  return b < p.nb && c == (unsigned)__ldg(p.cap + b) && lvl <= c;
}
__device__ __forceinline__ bool event_valid(const Params &p, const int4 &v) {
  unsigned meta = (unsigned)v.w;
  return (meta & 0xFFFFFu) < p.nc && ((meta >> 20) & 0x7FFu) < p.nk;
}

// region r of a call: 0 head (ts < t_begin), 1..W window r-1, W+1 tail (ts >= t_end[W-1])
struct Region {
  long long lo_ts, hi_ts;  // field-valid records of the region must satisfy lo <= ts < hi
  unsigned charge;         // window the region's drops are charged to
  int window;              // -1 for head / tail
};
__device__ __forceinline__ Region region_of(const Params &p, unsigned r) {
  Region g;
  if (r == 0) { g.lo_ts = kTsMin; g.hi_ts = p.T[0]; g.charge = 0; g.window = -1; }
  else if (r <= p.W) { g.lo_ts = p.T[r - 1]; g.hi_ts = p.T[r]; g.charge = r - 1; g.window = (int)r - 1; }
  else { g.lo_ts = p.T[p.W]; g.hi_ts = kTsMax; g.charge = p.W - 1; g.window = -1; }
  return g;
}

template <typename T>
__device__ __forceinline__ T warp_sum(T v) {
  for (int o = 16; o; o >>= 1) v += __shfl_xor_sync(kFull, v, o);
  return v;
}

// block-wide exclusive scan of one u32 per thread (blockDim.x <= 1024); returns exclusive prefix.
__device__ unsigned block_excl_scan(unsigned v, unsigned *scratch /*[32]*/, unsigned *total) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nw = (blockDim.x + 31) >> 5;
  unsigned x = v;
  for (int o = 1; o < 32; o <<= 1) {
    unsigned y = __shfl_up_sync(kFull, x, o);
    if (lane >= o) x += y;
  }
  if (lane == 31) scratch[warp] = x;
  __syncthreads();
  if (warp == 0) {
    unsigned s = lane < nw ? scratch[lane] : 0u;
    for (int o = 1; o < 32; o <<= 1) {
      unsigned y = __shfl_up_sync(kFull, s, o);
      if (lane >= o) s += y;
    }
    scratch[lane] = s;  // inclusive over warps
  }
  __syncthreads();
  unsigned base = warp ? scratch[warp - 1] : 0u;
  unsigned tot = scratch[nw - 1];
  __syncthreads();
  if (total) *total = tot;
  return base + x - v;
}

// ============================================================================================
// K0: region boundaries.  split(T) = smallest i such that every field-valid record at index
// >= i has ts >= T (= 1 + index of the last field-valid record with ts < T, or 0).  One warp
// per boundary, 33-ary search with 32 probes per step, then a linear warp scan.
// ============================================================================================
template <bool SAMPLES>
__global__ void k_split(Params p, long long *outB) {
  const unsigned q = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int lane = threadIdx.x & 31;
  if (q > p.W) return;
  const long long T = p.T[q];
  const unsigned long long N = SAMPLES ? p.ns : p.ne;
  const int4 *recs = SAMPLES ? reinterpret_cast<const int4 *>(p.s) : reinterpret_cast<const int4 *>(p.e);
  unsigned long long lo = 0, hi = N;
  while (hi - lo > 1024) {
    unsigned long long span = hi - lo;
    unsigned long long qq = lo + span * (unsigned long long)(lane + 1) / 33ull;
    int state = 0;  // 0 unknown, 1 valid with ts < T, 2 valid with ts >= T
    unsigned long long vpos = qq;
    for (int d = 0; d < 8; ++d) {
      unsigned long long i = qq + d;
      if (i >= hi) break;
      int4 v = __ldcg(recs + i);
      bool ok = SAMPLES ? sample_valid(p, v) : event_valid(p, v);
      if (ok) {
        state = rec_ts(v) >= T ? 2 : 1;
        vpos = i;
        break;
      }
    }
    unsigned long long nl = state == 1 ? vpos + 1 : lo;
    unsigned long long nh = state == 2 ? qq : hi;
    for (int o = 16; o; o >>= 1) {
      unsigned long long a = shfl_xor_ull(nl, o), b = shfl_xor_ull(nh, o);
      nl = a > nl ? a : nl;
      nh = b < nh ? b : nh;
    }
    if (nl == lo && nh == hi) break;  // only invalid records probed: fall back to the scan
    lo = nl;
    hi = nh < nl ? nl : nh;           // inconsistent only if unsorted (caught by the order check)
  }
  unsigned long long ans = lo;
  for (unsigned long long base = lo; base < hi; base += 32) {
    unsigned long long i = base + lane;
    bool pred = false;
    if (i < hi) {
      int4 v = __ldcg(recs + i);
      pred = (SAMPLES ? sample_valid(p, v) : event_valid(p, v)) && rec_ts(v) < T;
    }
    unsigned m = __ballot_sync(kFull, pred);
    if (m) ans = base + (unsigned long long)(32 - __clz(m));
  }
  if (lane == 0) outB[q] = (long long)ans;
}

__global__ void k_fill_tile_regions(const uint32_t *rt, uint32_t *tile_reg, uint32_t n_regions) {
  for (uint32_t r = blockIdx.x; r < n_regions; r += gridDim.x)
    for (uint32_t t = rt[r] + threadIdx.x; t < rt[r + 1]; t += blockDim.x) tile_reg[t] = r;
}

// ============================================================================================
// K1: sample partition.  One CTA per tile of <= 4096 samples of ONE region.  8 warps; warp w
// owns tile positions [512w, 512w+512), lane l handles positions 512w + 32j + l (j = 0..15),
// so each warp load is 512 contiguous bytes.  Kept samples are stably multisplit by bin
// (buffer_id >> 8): per-(warp, bin) running counters give a stable rank, a block scan gives
// bin offsets, the tile is permuted through shared memory and written out coalesced as
// 8-byte entries  ts_off<<24 | level<<8 | (buffer_id & 255).
// ============================================================================================
constexpr int kRecPerLane = kTileS / kK1Threads;  // 16
constexpr unsigned kNoKey = 0xFFFFu;

__global__ void __launch_bounds__(kK1Threads, 2) k_partition(Params p) {
  extern __shared__ __align__(16) unsigned char smem[];
  unsigned long long *sbuf = reinterpret_cast<unsigned long long *>(smem);                 // [4096]
  unsigned *binoff = reinterpret_cast<unsigned *>(sbuf + kTileS);                           // [nbins+1]
  unsigned short *cnt = reinterpret_cast<unsigned short *>(binoff + p.nbins + 1);          // [8][nbins]
  __shared__ unsigned scan_scratch[32];
  __shared__ long long wfirst[8], wlast[8];
  __shared__ unsigned whas[8], wviol[8], wkept[8];

  const unsigned tile = blockIdx.x;
  const unsigned r = p.tile_reg_s[tile];
  const long long start = p.Bs[r] + (long long)(tile - p.rts[r]) * kTileS;
  long long endp = p.Bs[r + 1];
  if (endp > start + kTileS) endp = start + kTileS;
  const int n = (int)(endp - start);
  const Region g = region_of(p, r);
  const bool is_win = g.window >= 0;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const unsigned lt = lanemask_lt();

  if (is_win)
    for (unsigned i = threadIdx.x; i < 8u * p.nbins; i += blockDim.x) cnt[i] = 0;
  __syncthreads();

  const int4 *src = reinterpret_cast<const int4 *>(p.s) + start;
  unsigned long long ent[kRecPerLane];
  unsigned kp[kRecPerLane];  // key << 16 | pos (kNoKey << 16: not kept)
  long long carry = kTsMin, first = kTsMax;
  bool has = false, viol = false;
  unsigned kept = 0;
#pragma unroll
  for (int h = 0; h < 2; ++h) {
    int4 v[8];
#pragma unroll
    for (int jj = 0; jj < 8; ++jj) {
      int i = warp * 512 + (h * 8 + jj) * 32 + lane;
      v[jj] = i < n ? ld_stream(src + i) : make_int4(0, 0, 0, 0);
    }
#pragma unroll
    for (int jj = 0; jj < 8; ++jj) {
      const int j = h * 8 + jj;
      const int i = warp * 512 + j * 32 + lane;
      const bool valid = i < n && sample_valid(p, v[jj]);
      const long long ts = rec_ts(v[jj]);
      const unsigned b = (unsigned)v[jj].z;
      // in-tile order: each field-valid record vs the previous field-valid record (warp order)
      const unsigned vm = __ballot_sync(kFull, valid);
      const unsigned lower = vm & lt;
      const long long prev = shfl_ll(ts, lower ? 31 - __clz(lower) : lane);
      if (valid && ((lower ? prev : carry) > ts || ts < g.lo_ts || ts >= g.hi_ts)) viol = true;
      if (vm) {
        if (!has) first = shfl_ll(ts, __ffs(vm) - 1);
        has = true;
        carry = shfl_ll(ts, 31 - __clz(vm));
      }
      const bool keep = valid && is_win;
      kept += keep;
      unsigned key = keep ? (b >> kBinLog) : kNoKey;
      unsigned pos = 0;
      if (is_win) {
        const unsigned peers = __match_any_sync(kFull, key);
        unsigned basec = 0;
        if (keep) basec = cnt[warp * p.nbins + key];
        __syncwarp();
        if (keep && lane == __ffs(peers) - 1) cnt[warp * p.nbins + key] = (unsigned short)(basec + __popc(peers));
        __syncwarp();
        pos = basec + __popc(peers & lt);
        ent[j] = ((unsigned long long)(ts - g.lo_ts) << 24) |
                 ((unsigned long long)((unsigned)v[jj].w & 0xFFFFu) << 8) | (b & (kBin - 1));
      }
      kp[j] = (key << 16) | pos;
    }
  }
  // warp summaries -> tile summary
  kept = warp_sum(kept);
  const bool wv = __any_sync(kFull, viol);
  if (lane == 0) {
    wfirst[warp] = first;
    wlast[warp] = carry;
    whas[warp] = has;
    wviol[warp] = wv;
    wkept[warp] = kept;
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    long long run = kTsMin, tf = 0;
    bool th = false, tv = false;
    unsigned tk = 0;
    for (int w = 0; w < 8; ++w) {
      tk += wkept[w];
      tv |= wviol[w] != 0;
      if (whas[w]) {
        if (wfirst[w] < run) tv = true;
        if (!th) tf = wfirst[w];
        th = true;
        run = wlast[w];
      }
    }
    TileMeta m;
    m.first_ts = tf;
    m.last_ts = run;
    m.flags = (th ? 1u : 0u) | (tv ? 2u : 0u);
    m.pad = 0;
    p.smeta[tile] = m;
    if ((unsigned)n > tk) atomicAdd(p.win + WF_DROPPED * p.W + g.charge, (unsigned long long)(n - tk));
    if (tk) atomicAdd(p.win + WF_SAMPLES * p.W + g.window, (unsigned long long)tk);
    wkept[0] = tk;
  }
  if (!is_win) return;
  __syncthreads();
  const unsigned total_kept = wkept[0];

  // per-bin exclusive prefix over warps, bin totals, exclusive scan over bins
  const unsigned nb = p.nbins;
  const unsigned chunk = (nb + blockDim.x - 1) / blockDim.x;
  const unsigned b0 = threadIdx.x * chunk;
  unsigned csum = 0;
  for (unsigned bb = b0; bb < b0 + chunk && bb < nb; ++bb) {
    unsigned run = 0;
    for (int w = 0; w < 8; ++w) {
      unsigned c = cnt[w * nb + bb];
      cnt[w * nb + bb] = (unsigned short)run;
      run += c;
    }
    binoff[bb] = run;
    csum += run;
  }
  unsigned base = block_excl_scan(csum, scan_scratch, nullptr);
  for (unsigned bb = b0; bb < b0 + chunk && bb < nb; ++bb) {
    unsigned t = binoff[bb];
    binoff[bb] = base;
    base += t;
  }
  if (threadIdx.x == 0) binoff[nb] = total_kept;
  __syncthreads();
  uint32_t *offs = p.soff + (size_t)tile * (nb + 1);
  for (unsigned bb = threadIdx.x; bb <= nb; bb += blockDim.x) offs[bb] = binoff[bb];
#pragma unroll
  for (int j = 0; j < kRecPerLane; ++j) {
    unsigned key = kp[j] >> 16;
    if (key != kNoKey) sbuf[binoff[key] + cnt[warp * nb + key] + (kp[j] & 0xFFFFu)] = ent[j];
  }
  __syncthreads();
  unsigned long long *dst = p.stage + (size_t)tile * kTileS;
  for (unsigned i = threadIdx.x; i < total_kept; i += blockDim.x) dst[i] = sbuf[i];
}

// ============================================================================================
// K3: task events.  One CTA per tile of <= 4096 events of one region: validate, order-check,
// per-(window, kernel) START/END counts, per-(window, component) activity bits and per-call
// per-component START/END deltas (progress bars, L131; "task counts stop changing", L227).
// ============================================================================================
__global__ void __launch_bounds__(kK3Threads) k_events(Params p) {
  extern __shared__ __align__(16) unsigned char smem[];
  unsigned *khist = reinterpret_cast<unsigned *>(smem);  // [nk*2]
  unsigned *abits = khist + 2 * p.nk;                     // [ncw] if smem_bits
  __shared__ long long wfirst[8], wlast[8];
  __shared__ unsigned whas[8], wviol[8], wkept[8];
  const bool smem_bits = p.ncw <= 2048;

  const unsigned tile = blockIdx.x;
  const unsigned r = p.tile_reg_e[tile];
  const long long start = p.Be[r] + (long long)(tile - p.rte[r]) * kTileE;
  long long endp = p.Be[r + 1];
  if (endp > start + kTileE) endp = start + kTileE;
  const int n = (int)(endp - start);
  const Region g = region_of(p, r);
  const bool is_win = g.window >= 0;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const unsigned lt = lanemask_lt();
  if (is_win) {
    for (unsigned i = threadIdx.x; i < 2 * p.nk; i += blockDim.x) khist[i] = 0;
    if (smem_bits)
      for (unsigned i = threadIdx.x; i < p.ncw; i += blockDim.x) abits[i] = 0;
  }
  __syncthreads();
  const int4 *src = reinterpret_cast<const int4 *>(p.e) + start;
  long long carry = kTsMin, first = kTsMax;
  bool has = false, viol = false;
  unsigned kept = 0;
#pragma unroll
  for (int h = 0; h < 2; ++h) {
    int4 v[8];
#pragma unroll
    for (int jj = 0; jj < 8; ++jj) {
      int i = warp * 512 + (h * 8 + jj) * 32 + lane;
      v[jj] = i < n ? ld_stream(src + i) : make_int4(0, 0, 0, 0);
    }
#pragma unroll
    for (int jj = 0; jj < 8; ++jj) {
      const int i = warp * 512 + (h * 8 + jj) * 32 + lane;
      const bool valid = i < n && event_valid(p, v[jj]);
      const long long ts = rec_ts(v[jj]);
      const unsigned vm = __ballot_sync(kFull, valid);
      const unsigned lower = vm & lt;
      const long long prev = shfl_ll(ts, lower ? 31 - __clz(lower) : lane);
      if (valid && ((lower ? prev : carry) > ts || ts < g.lo_ts || ts >= g.hi_ts)) viol = true;
      if (vm) {
        if (!has) first = shfl_ll(ts, __ffs(vm) - 1);
        has = true;
        carry = shfl_ll(ts, 31 - __clz(vm));
      }
      const bool keep = valid && is_win;
      kept += keep;
      const unsigned meta = (unsigned)v[jj].w;
      const unsigned comp = meta & 0xFFFFFu, kern = (meta >> 20) & 0x7FFu, kind = meta >> 31;
      const unsigned kk = keep ? kern * 2 + kind : 0xFFFFFFFFu;
      const unsigned peers = __match_any_sync(kFull, kk);
      if (keep && lane == __ffs(peers) - 1) atomicAdd(&khist[kk], (unsigned)__popc(peers));
      if (keep) {
        if (smem_bits) atomicOr(&abits[comp >> 5], 1u << (comp & 31));
        else atomicOr(p.active + (size_t)g.window * p.ncw + (comp >> 5), 1u << (comp & 31));
        atomicAdd(p.cdelta + 2 * comp + kind, 1ull);
      }
    }
  }
  kept = warp_sum(kept);
  const bool wv = __any_sync(kFull, viol);
  if (lane == 0) {
    wfirst[warp] = first;
    wlast[warp] = carry;
    whas[warp] = has;
    wviol[warp] = wv;
    wkept[warp] = kept;
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    long long run = kTsMin, tf = 0;
    bool th = false, tv = false;
    unsigned tk = 0;
    for (int w = 0; w < 8; ++w) {
      tk += wkept[w];
      tv |= wviol[w] != 0;
      if (whas[w]) {
        if (wfirst[w] < run) tv = true;
        if (!th) tf = wfirst[w];
        th = true;
        run = wlast[w];
      }
    }
    TileMeta m;
    m.first_ts = tf;
    m.last_ts = run;
    m.flags = (th ? 1u : 0u) | (tv ? 2u : 0u);
    m.pad = 0;
    p.emeta[tile] = m;
    if ((unsigned)n > tk) atomicAdd(p.win + WF_DROPPED * p.W + g.charge, (unsigned long long)(n - tk));
    if (tk) atomicAdd(p.win + WF_EVENTS * p.W + g.window, (unsigned long long)tk);
  }
  if (!is_win) return;
  for (unsigned i = threadIdx.x; i < 2 * p.nk; i += blockDim.x)
    if (khist[i]) atomicAdd(p.kdelta + ((size_t)g.window * p.nk) * 2 + i, khist[i]);
  if (smem_bits)
    for (unsigned i = threadIdx.x; i < p.ncw; i += blockDim.x)
      if (abits[i]) atomicOr(p.active + (size_t)g.window * p.ncw + i, abits[i]);
}

// ============================================================================================
// K2: fold.  One warp per (window, bin) unit; units are dequeued in window-major order, so a
// unit only ever waits on units dequeued before it (forward progress).  Phase 1 folds the
// bin's kept samples in ingest order with the carry-in left symbolic:
//     I = L_in * (ts_0 - t_begin) + D,   D = sum_i (l_i - l_{i-1}) * (t_end - ts_i), l_{-1} = 0
// (telescoping form of sum level*dt; D needs only each sample's predecessor level, found with
// __match_any_sync inside a 32-sample step and in shared memory across steps).  It then
// publishes the window's last levels (kSent for untouched buffers) and a flag.  Phase 2 gets
// L_in from the nearest earlier window with a resolved level (decoupled look-back), finalizes
// and resolves its own untouched cells.
// ============================================================================================
struct FoldSmem {
  unsigned long long D[kBin];
  unsigned long long ts0[kBin];
  unsigned n[kBin];
  unsigned short cur[kBin], pmax[kBin], pmin[kBin];
  unsigned long long sc[32];
  unsigned short sl[32];
};

__global__ void __launch_bounds__(kFoldWarps * 32) k_fold(Params p) {
  extern __shared__ __align__(16) unsigned char smem[];
  FoldSmem &S = reinterpret_cast<FoldSmem *>(smem)[threadIdx.x >> 5];
  const int lane = threadIdx.x & 31;
  const unsigned lt = lanemask_lt();
  const unsigned n_units = p.W * p.nbins;
  for (;;) {
    unsigned u = 0;
    if (lane == 0) u = atomicAdd(p.unit_ctr, 1u);
    u = __shfl_sync(kFull, u, 0);
    if (u >= n_units) break;
    const unsigned w = u / p.nbins, bin = u % p.nbins;
    const long long tb = p.T[w], te = p.T[w + 1];
    const unsigned long long Wlen = (unsigned long long)(te - tb);
    const unsigned t_lo = p.rts[w + 1], t_hi = p.rts[w + 2];
#pragma unroll
    for (int i = 0; i < kBin / 32; ++i) {
      const int l = lane + 32 * i;
      S.D[l] = 0;
      S.n[l] = 0;
      S.cur[l] = 0;
      S.pmax[l] = 0;
      S.pmin[l] = 0xFFFFu;
    }
    __syncwarp();
    // ---- phase 1: in-order fold over the (tile, bin) segments of window w
    for (unsigned tg = t_lo; tg < t_hi; tg += 32) {
      unsigned seg_lo = 0, seg_len = 0;
      if (tg + lane < t_hi) {
        const uint32_t *o = p.soff + (size_t)(tg + lane) * (p.nbins + 1) + bin;
        seg_lo = __ldg(o);
        seg_len = __ldg(o + 1) - seg_lo;
      }
      const unsigned nseg = min(32u, t_hi - tg);
      for (unsigned sg = 0; sg < nseg; ++sg) {
        const unsigned lo = __shfl_sync(kFull, seg_lo, sg), len = __shfl_sync(kFull, seg_len, sg);
        const unsigned long long *seg = p.stage + (size_t)(tg + sg) * kTileS + lo;
        for (unsigned c = 0; c < len; c += 32) {
          const bool act = c + lane < len;
          const unsigned long long e = act ? __ldcg(seg + c + lane) : 0ull;
          const unsigned lid = act ? (unsigned)(e & (kBin - 1)) : (unsigned)(kBin + lane);
          const unsigned lvl = (unsigned)(e >> 8) & 0xFFFFu;
          const unsigned long long off = e >> 24;
          const unsigned peers = __match_any_sync(kFull, lid);
          const unsigned lower = peers & lt;
          const unsigned plv = __shfl_sync(kFull, lvl, lower ? 31 - __clz(lower) : lane);
          unsigned long long contrib = 0;
          if (act) {
            unsigned prev;
            if (lower) {
              prev = plv;
            } else {
              prev = S.cur[lid];
              if (S.n[lid] == 0) S.ts0[lid] = off;
            }
            contrib = (unsigned long long)((long long)((int)lvl - (int)prev) * (long long)(Wlen - off));
          }
          S.sc[lane] = contrib;
          S.sl[lane] = (unsigned short)lvl;
          __syncwarp();
          if (act && (peers >> lane) == 1u) {  // last lane of its group applies the group
            unsigned long long sum = 0;
            unsigned mx = 0, mn = 0xFFFFu;
            unsigned m = peers;
            while (m) {
              const int j = __ffs(m) - 1;
              m &= m - 1;
              sum += S.sc[j];
              const unsigned x = S.sl[j];
              mx = x > mx ? x : mx;
              mn = x < mn ? x : mn;
            }
            S.D[lid] += sum;
            S.n[lid] += __popc(peers);
            S.cur[lid] = (unsigned short)lvl;
            if (mx > S.pmax[lid]) S.pmax[lid] = (unsigned short)mx;
            if (mn < S.pmin[lid]) S.pmin[lid] = (unsigned short)mn;
          }
          __syncwarp();
        }
      }
    }
    // ---- publish this window's last levels (kSent: untouched) and the phase-1 flag
    const unsigned b_base = bin * kBin;
    uint16_t *lw = p.lastlvl + (size_t)w * p.nb;
#pragma unroll
    for (int i = 0; i < kBin / 32; ++i) {
      const unsigned l = lane + 32 * i, b = b_base + l;
      if (b < p.nb) lw[b] = S.n[l] ? S.cur[l] : kSent;
    }
    __threadfence();
    __syncwarp();
    if (lane == 0) st_release_u32(p.flags + (size_t)w * p.nbins + bin, p.epoch);
    // ---- phase 2: carry-in by look-back, finalize
    unsigned short lin[kBin / 32];
    unsigned need = 0;
#pragma unroll
    for (int i = 0; i < kBin / 32; ++i) {
      lin[i] = 0;
      if (b_base + lane + 32 * i < p.nb) need |= 1u << i;
    }
    int j = (int)w - 1;
    while (__any_sync(kFull, need != 0)) {
      if (j < 0) {
#pragma unroll
        for (int i = 0; i < kBin / 32; ++i)
          if (need & (1u << i)) lin[i] = __ldg(p.carry_in + b_base + lane + 32 * i);
        need = 0;
        break;
      }
      if (lane == 0) {
        const unsigned *f = p.flags + (size_t)j * p.nbins + bin;
        unsigned spins = 0;
        while (ld_acquire_u32(f) != p.epoch) {
          __nanosleep(64);
          if (++spins > (1u << 25)) {  // ~seconds: never expected; fail loudly instead of hanging
            atomicOr(p.status, 4u);
            break;
          }
        }
      }
      __syncwarp();
      const unsigned short *lj = p.lastlvl + (size_t)j * p.nb + b_base + lane;
#pragma unroll
      for (int i = 0; i < kBin / 32; ++i) {
        if (need & (1u << i)) {
          const unsigned short v = ld_relaxed_u16(lj + 32 * i);
          if (v != kSent) {
            lin[i] = v;
            need &= ~(1u << i);
          }
        }
      }
      --j;
    }
    unsigned long long dig = 0;
    unsigned touched = 0;
    const bool last_window = (w == p.W - 1);
#pragma unroll
    for (int i = 0; i < kBin / 32; ++i) {
      const unsigned l = lane + 32 * i, b = b_base + l;
      if (b >= p.nb) continue;
      const unsigned L = lin[i];
      const unsigned cnt = S.n[l];
      unsigned long long I;
      unsigned mx, mn, last;
      if (cnt) {
        I = (unsigned long long)L * S.ts0[l] + S.D[l];
        mx = S.pmax[l] > L ? S.pmax[l] : L;
        mn = S.pmin[l] < L ? S.pmin[l] : L;
        last = S.cur[l];
      } else {
        I = (unsigned long long)L * Wlen;
        mx = mn = last = L;
        lw[b] = (uint16_t)L;  // resolve the untouched cell
      }
      const unsigned capb = __ldg(p.cap + b);
      if (mn == capb) {
        const unsigned c = __ldg(p.owner + b);
        atomicOr(p.anyfull + (size_t)w * p.ncw + (c >> 5), 1u << (c & 31));
      }
      if (cnt) {
        // digest term: splitmix64 finalizer absorbed four times
        auto fm = [](unsigned long long z) {
          z ^= z >> 30;
          z *= 0xbf58476d1ce4e5b9ULL;
          z ^= z >> 27;
          z *= 0x94d049bb133111ebULL;
          z ^= z >> 31;
          return z;
        };
        unsigned long long h = fm(0x9E3779B97F4A7C15ULL ^ (unsigned long long)b);
        h = fm(h ^ ((unsigned long long)last | ((unsigned long long)mx << 16) | ((unsigned long long)mn << 32) |
                    ((unsigned long long)capb << 48)));
        h = fm(h ^ (unsigned long long)cnt);
        h = fm(h ^ I);
        dig += h;
        ++touched;
      }
      if (last_window) {
        rtm_buffer_stat st;
        st.integral = (int64_t)I;
        st.last = (uint16_t)last;
        st.max = (uint16_t)mx;
        st.min = (uint16_t)mn;
        st.capacity = (uint16_t)capb;
        st.n_samples = cnt;
        st.reserved = __ldg(p.elig + b);
        st.mean_occ = Wlen ? __ddiv_rn((double)(long long)I, (double)((long long)capb * (long long)Wlen)) : 0.0;
        p.bstat[b] = st;
        p.carry_out[b] = (uint16_t)last;
      }
    }
    dig = warp_sum(dig);
    touched = warp_sum(touched);
    if (lane == 0) {
      if (dig) atomicAdd(p.win + WF_DIGEST * p.W + w, dig);
      if (touched) atomicAdd(p.win + WF_TOUCHED * p.W + w, (unsigned long long)touched);
    }
    __syncwarp();
  }
}

// ============================================================================================
// K4: cross-tile order check (single CTA).  Tile t violates the contract if its own flag is set
// or its first field-valid ts is below the max ts of all earlier tiles.
// ============================================================================================
__global__ void __launch_bounds__(1024) k_order_check(const TileMeta *meta, unsigned n, unsigned *status,
                                                       unsigned bit) {
  __shared__ long long wmax[32];
  __shared__ long long carry_s;
  __shared__ unsigned bad_s;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  if (threadIdx.x == 0) { carry_s = kTsMin; bad_s = 0; }
  __syncthreads();
  for (unsigned base = 0; base < n; base += blockDim.x) {
    const unsigned t = base + threadIdx.x;
    TileMeta m;
    m.flags = 0; m.first_ts = 0; m.last_ts = kTsMin;
    if (t < n) m = meta[t];
    const bool has = m.flags & 1u;
    long long x = has ? m.last_ts : kTsMin;  // inclusive max-scan
    for (int o = 1; o < 32; o <<= 1) {
      long long y = shfl_ll(x, lane >= o ? lane - o : lane);
      if (lane >= o && y > x) x = y;
    }
    if (lane == 31) wmax[warp] = x;
    __syncthreads();
    if (warp == 0) {
      long long s = wmax[lane];
      for (int o = 1; o < 32; o <<= 1) {
        long long y = shfl_ll(s, lane >= o ? lane - o : lane);
        if (lane >= o && y > s) s = y;
      }
      wmax[lane] = s;
    }
    __syncthreads();
    long long before = carry_s;
    const long long wprev = warp ? wmax[warp - 1] : kTsMin;
    if (wprev > before) before = wprev;
    long long xin = shfl_ll(x, lane ? lane - 1 : 0);
    if (lane && xin > before) before = xin;
    bool bad = (m.flags & 2u) || (has && m.first_ts < before);
    if (__any_sync(kFull, bad) && lane == 0) atomicOr(&bad_s, 1u);
    __syncthreads();
    if (threadIdx.x == 0 && wmax[31] > carry_s) carry_s = wmax[31];
    __syncthreads();
  }
  if (threadIdx.x == 0 && bad_s) atomicOr(status, bit);
}

// ============================================================================================
// K5: top-k (Bottleneck Analyzer list).  One CTA per window.  Fullness key:
// key32 = 0xFFFFFFFF if level == cap else floor(level * 2^32 / cap), exactly order-preserving
// for cap <= 65535; size mode key32 = level.  MSB-first radix select (4 x 8
// bits) finds the k-th key tau; keys > tau are taken, keys == tau are taken in buffer_id order
// (tie-break), and the k winners are bitonic-sorted by (key desc, id asc).
// ============================================================================================
constexpr int kTopkThreads = 512;

__device__ __forceinline__ unsigned fullness_key(unsigned l, unsigned c, int mode) {
  if (mode == RTM_RANK_SIZE) return l;
  if (l == c) return 0xFFFFFFFFu;
  return (unsigned)(((unsigned long long)l << 32) / c);
}

__global__ void __launch_bounds__(kTopkThreads) k_topk(Params p) {
  extern __shared__ __align__(16) unsigned char smem[];
  const unsigned nb = p.nb;
  const bool keys_in_smem = nb <= kTopkSmemKeys;
  unsigned *keys = reinterpret_cast<unsigned *>(smem);                                  // [nb] or none
  unsigned *hist = keys + (keys_in_smem ? ((nb + 1) & ~1u) : 0);                        // [16][256]
  unsigned long long *sel = reinterpret_cast<unsigned long long *>(hist + 16 * 256);    // [1024]
  __shared__ unsigned scan_scratch[32];
  __shared__ unsigned s_digit, s_need, s_ngt;
  const unsigned w = blockIdx.x;
  const uint16_t *lv = p.lastlvl + (size_t)w * nb;
  const int warp = threadIdx.x >> 5;

  auto key_of = [&](unsigned b, bool &el) -> unsigned {
    el = __ldg(p.elig + b) != 0;
    return fullness_key(lv[b], __ldg(p.cap + b), p.rank_mode);
  };
  unsigned n_el = 0;
  if (keys_in_smem) {
    for (unsigned b = threadIdx.x; b < nb; b += blockDim.x) {
      bool el;
      unsigned k = key_of(b, el);
      keys[b] = k;
      n_el += el;
    }
  } else {
    for (unsigned b = threadIdx.x; b < nb; b += blockDim.x) n_el += __ldg(p.elig + b) != 0;
  }
  unsigned tot_el;
  block_excl_scan(n_el, scan_scratch, &tot_el);
  const unsigned keff = p.k < tot_el ? p.k : tot_el;
  if (keff == 0) {
    if (threadIdx.x == 0) p.topk_n[w] = 0;
    return;
  }
  unsigned prefix = 0, mask = 0, need = keff;
  for (int d = 3; d >= 0; --d) {
    for (unsigned i = threadIdx.x; i < 16 * 256; i += blockDim.x) hist[i] = 0;
    __syncthreads();
    unsigned *myh = hist + (warp & 15) * 256;
    for (unsigned b = threadIdx.x; b < nb; b += blockDim.x) {
      bool el;
      unsigned k;
      if (keys_in_smem) { k = keys[b]; el = __ldg(p.elig + b) != 0; }
      else k = key_of(b, el);
      if (el && (k & mask) == prefix) atomicAdd(&myh[(k >> (8 * d)) & 255u], 1u);
    }
    __syncthreads();
    if (threadIdx.x < 256) {
      unsigned s = 0;
      for (int q = 0; q < 16; ++q) s += hist[q * 256 + threadIdx.x];
      hist[threadIdx.x] = s;  // row 0 now holds totals (rows read before overwrite by owner only)
    }
    __syncthreads();
    if (threadIdx.x == 0) {
      unsigned cum = 0;
      int x = 255;
      for (; x > 0; --x) {
        if (cum + hist[x] >= need) break;
        cum += hist[x];
      }
      s_digit = (unsigned)x;
      s_need = need - cum;
    }
    __syncthreads();
    prefix |= s_digit << (8 * d);
    mask |= 255u << (8 * d);
    need = s_need;
    __syncthreads();
  }
  const unsigned tau = prefix;  // k-th key; `need` keys equal to tau are taken (lowest ids)
  if (threadIdx.x == 0) s_ngt = 0;
  __syncthreads();
  // keys > tau (count keff - need), any order
  for (unsigned b = threadIdx.x; b < nb; b += blockDim.x) {
    bool el;
    unsigned k;
    if (keys_in_smem) { k = keys[b]; el = __ldg(p.elig + b) != 0; }
    else k = key_of(b, el);
    if (el && k > tau) {
      unsigned slot = atomicAdd(&s_ngt, 1u);
      sel[slot] = ((unsigned long long)k << 32) | (0xFFFFFFFFu - b);
    }
  }
  __syncthreads();
  const unsigned ngt = s_ngt;
  // keys == tau in id order: contiguous id chunk per thread, block scan for stable ranks
  const unsigned chunk = (nb + blockDim.x - 1) / blockDim.x;
  const unsigned c0 = threadIdx.x * chunk;
  unsigned ceq = 0;
  for (unsigned b = c0; b < c0 + chunk && b < nb; ++b) {
    bool el;
    unsigned k;
    if (keys_in_smem) { k = keys[b]; el = __ldg(p.elig + b) != 0; }
    else k = key_of(b, el);
    ceq += (el && k == tau);
  }
  unsigned rank = block_excl_scan(ceq, scan_scratch, nullptr);
  for (unsigned b = c0; b < c0 + chunk && b < nb && rank < need; ++b) {
    bool el;
    unsigned k;
    if (keys_in_smem) { k = keys[b]; el = __ldg(p.elig + b) != 0; }
    else k = key_of(b, el);
    if (el && k == tau) {
      sel[ngt + rank] = ((unsigned long long)k << 32) | (0xFFFFFFFFu - b);
      ++rank;
    }
  }
  __syncthreads();
  // bitonic sort descending over the next power of two >= keff
  unsigned P = 1;
  while (P < keff) P <<= 1;
  for (unsigned i = keff + threadIdx.x; i < P; i += blockDim.x) sel[i] = 0ull;
  __syncthreads();
  for (unsigned size = 2; size <= P; size <<= 1) {
    for (unsigned stride = size >> 1; stride > 0; stride >>= 1) {
      for (unsigned i = threadIdx.x; i < P; i += blockDim.x) {
        unsigned jx = i ^ stride;
        if (jx > i) {
          bool desc = (i & size) == 0;
          unsigned long long a = sel[i], b = sel[jx];
          if ((a < b) == desc) { sel[i] = b; sel[jx] = a; }
        }
      }
      __syncthreads();
    }
  }
  for (unsigned i = threadIdx.x; i < p.k; i += blockDim.x) {
    unsigned long long out = 0xFFFFFFFFull;  // buffer_id 0xFFFFFFFF, level 0, cap 0
    if (i < keff) {
      unsigned b = 0xFFFFFFFFu - (unsigned)(sel[i] & 0xFFFFFFFFu);
      out = (unsigned long long)b | ((unsigned long long)lv[b] << 32) | ((unsigned long long)__ldg(p.cap + b) << 48);
    }
    p.topk[(size_t)w * p.k + i] = out;
  }
  if (threadIdx.x == 0) p.topk_n[w] = keff;
}

// ============================================================================================
// K6: hang flag (L227-L229): cond_c(w) = any buffer of c full for the whole window AND no task
// event of c in w; run_c counts consecutive cond windows; flagged when run_c >= H.
// One thread per component; a warp covers one 32-component bitmap word.
// ============================================================================================
__global__ void k_hang(Params p) {
  const unsigned c = blockIdx.x * blockDim.x + threadIdx.x;
  const unsigned word = c >> 5, bit = c & 31;
  const bool in = c < p.nc;
  unsigned run = in ? p.run[c] : 0u;
  const bool wordok = word < p.ncw;
  for (unsigned w = 0; w < p.W; ++w) {
    unsigned f = 0, a = 0;
    if (wordok) {
      f = __ldg(p.anyfull + (size_t)w * p.ncw + word);
      a = __ldg(p.active + (size_t)w * p.ncw + word);
    }
    const bool cond = in && ((f >> bit) & 1u) && !((a >> bit) & 1u);
    run = cond ? run + 1 : 0u;
    const unsigned fl = __ballot_sync(kFull, in && run >= p.H);
    if ((threadIdx.x & 31) == 0 && wordok) {
      p.hung[(size_t)w * p.ncw + word] = fl;
      if (fl) atomicAdd(p.win + WF_HUNG * p.W + w, (unsigned long long)__popc(fl));
    }
  }
  if (in) p.run[c] = run;
}

// ============================================================================================
// K7: progress bars (L131): per kernel, cumulative START/END over windows (block scan), and
// the per-component cumulative counts for the last window.
// ============================================================================================
__global__ void __launch_bounds__(256) k_progress(Params p) {
  __shared__ unsigned scan_scratch[32];
  const unsigned k = blockIdx.x;
  if (k < p.nk) {
    long long s = p.kstart[k], e = p.kend[k];
    const long long total = p.ktotal[k];
    for (unsigned base = 0; base < p.W; base += blockDim.x) {
      const unsigned w = base + threadIdx.x;
      unsigned ds = 0, de = 0;
      if (w < p.W) {
        ds = p.kdelta[((size_t)w * p.nk + k) * 2 + 0];
        de = p.kdelta[((size_t)w * p.nk + k) * 2 + 1];
      }
      unsigned ts_, te_;
      unsigned xs = block_excl_scan(ds, scan_scratch, &ts_);
      unsigned xe = block_excl_scan(de, scan_scratch, &te_);
      if (w < p.W) {
        long long S = s + xs + ds, E = e + xe + de;
        long long *o = p.prog + ((size_t)w * p.nk + k) * 5;
        o[0] = total;
        o[1] = S;
        o[2] = E;
        o[3] = S - E;
        o[4] = total - S;
      }
      s += ts_;
      e += te_;
    }
    if (threadIdx.x == 0) {
      p.kstart[k] = s;
      p.kend[k] = e;
    }
  } else {
    for (unsigned c = (k - p.nk) * blockDim.x + threadIdx.x; c < p.nc; c += (gridDim.x - p.nk) * blockDim.x) {
      long long s = p.cstart[c] + (long long)p.cdelta[2 * c], e = p.cend[c] + (long long)p.cdelta[2 * c + 1];
      p.cstart[c] = s;
      p.cend[c] = e;
      rtm_component_tasks t;
      t.started = s;
      t.finished = e;
      t.in_flight = s - e;
      p.comps[c] = t;
    }
  }
}

// ============================================================================================
// Multi-rank merge (world > 1).  Pack layout per rank (bytes, 8-aligned sections):
//   win [kWinFields][W] u64 | topk [W][k] u64 | topk_n [W] u32 (padded) | prog [W][nk][5] i64 |
//   hung [W][ncw] u32 (padded) | comps [nc] (3 x i64) | bstat [nb] (32 B; reserved = owned)
// ============================================================================================
struct PackLayout {
  size_t win, topk, topk_n, prog, hung, comps, bstat, total;
};
__host__ __device__ inline size_t align8(size_t x) { return (x + 7) & ~(size_t)7; }
__host__ __device__ inline PackLayout pack_layout(const Params &p) {
  PackLayout L;
  size_t o = 0;
  L.win = o; o += align8((size_t)kWinFields * p.W * 8);
  L.topk = o; o += align8((size_t)p.W * p.k * 8);
  L.topk_n = o; o += align8((size_t)p.W * 4);
  L.prog = o; o += align8((size_t)p.W * p.nk * 5 * 8);
  L.hung = o; o += align8((size_t)p.W * p.ncw * 4);
  L.comps = o; o += align8((size_t)p.nc * sizeof(rtm_component_tasks));
  L.bstat = o; o += align8((size_t)p.nb * sizeof(rtm_buffer_stat));
  L.total = o;
  return L;
}

__device__ __forceinline__ unsigned long long topk_composite(unsigned long long ent, int mode) {
  const unsigned b = (unsigned)(ent & 0xFFFFFFFFu);
  const unsigned l = (unsigned)(ent >> 32) & 0xFFFFu, c = (unsigned)(ent >> 48);
  return ((unsigned long long)fullness_key(l, c, mode) << 32) | (0xFFFFFFFFu - b);
}

// one CTA per window: merge world x k candidates; sums of scalar fields; progress sums; hang OR
__global__ void __launch_bounds__(256) k_merge_windows(Params p, const unsigned char *g, unsigned world,
                                                       size_t stride) {
  extern __shared__ __align__(16) unsigned char smem[];
  unsigned long long *cand = reinterpret_cast<unsigned long long *>(smem);  // [P] composite keys
  const PackLayout L = pack_layout(p);
  const unsigned w = blockIdx.x;
  const unsigned nc_all = world * p.k;
  unsigned P = 1;
  while (P < nc_all) P <<= 1;
  unsigned long long *full_ent = cand + P;  // [P] entries aligned with cand
  for (unsigned i = threadIdx.x; i < P; i += blockDim.x) {
    unsigned long long key = 0, en = 0;
    if (i < nc_all) {
      const unsigned r = i / p.k, s = i % p.k;
      const unsigned char *base = g + stride * r;
      const unsigned n = reinterpret_cast<const unsigned *>(base + L.topk_n)[w];
      if (s < n) {
        en = reinterpret_cast<const unsigned long long *>(base + L.topk)[(size_t)w * p.k + s];
        key = topk_composite(en, p.rank_mode);
      }
    }
    cand[i] = key;
    full_ent[i] = en;
  }
  __syncthreads();
  for (unsigned size = 2; size <= P; size <<= 1) {
    for (unsigned stride2 = size >> 1; stride2 > 0; stride2 >>= 1) {
      for (unsigned i = threadIdx.x; i < P; i += blockDim.x) {
        unsigned jx = i ^ stride2;
        if (jx > i) {
          bool desc = (i & size) == 0;
          unsigned long long a = cand[i], b = cand[jx];
          if ((a < b) == desc) {
            cand[i] = b; cand[jx] = a;
            unsigned long long t = full_ent[i]; full_ent[i] = full_ent[jx]; full_ent[jx] = t;
          }
        }
      }
      __syncthreads();
    }
  }
  __shared__ unsigned s_n;
  if (threadIdx.x == 0) {
    unsigned n = 0;
    for (unsigned r = 0; r < world; ++r) n += reinterpret_cast<const unsigned *>(g + stride * r + L.topk_n)[w];
    s_n = n < p.k ? n : p.k;
    p.topk_n[w] = s_n;
  }
  __syncthreads();
  for (unsigned i = threadIdx.x; i < p.k; i += blockDim.x)
    p.topk[(size_t)w * p.k + i] = i < s_n ? full_ent[i] : 0xFFFFFFFFull;
  // scalar fields
  if (threadIdx.x < kWinFields) {
    unsigned long long s = 0;
    for (unsigned r = 0; r < world; ++r)
      s += reinterpret_cast<const unsigned long long *>(g + stride * r + L.win)[(size_t)threadIdx.x * p.W + w];
    p.win[(size_t)threadIdx.x * p.W + w] = s;
  }
  // progress: sum of per-rank cumulative START / END
  for (unsigned k = threadIdx.x; k < p.nk; k += blockDim.x) {
    long long S = 0, E = 0;
    for (unsigned r = 0; r < world; ++r) {
      const long long *o = reinterpret_cast<const long long *>(g + stride * r + L.prog) + ((size_t)w * p.nk + k) * 5;
      S += o[1];
      E += o[2];
    }
    long long *o = p.prog + ((size_t)w * p.nk + k) * 5;
    const long long total = p.ktotal[k];
    o[0] = total; o[1] = S; o[2] = E; o[3] = S - E; o[4] = total - S;
  }
  for (unsigned q = threadIdx.x; q < p.ncw; q += blockDim.x) {
    unsigned x = 0;
    for (unsigned r = 0; r < world; ++r) x |= reinterpret_cast<const unsigned *>(g + stride * r + L.hung)[(size_t)w * p.ncw + q];
    p.hung[(size_t)w * p.ncw + q] = x;
  }
}

__global__ void k_merge_tables(Params p, const unsigned char *g, unsigned world, size_t stride) {
  const PackLayout L = pack_layout(p);
  const size_t tid = (size_t)blockIdx.x * blockDim.x + threadIdx.x, nth = (size_t)gridDim.x * blockDim.x;
  for (size_t c = tid; c < p.nc; c += nth) {
    rtm_component_tasks t = {0, 0, 0};
    for (unsigned r = 0; r < world; ++r) {
      const rtm_component_tasks x = reinterpret_cast<const rtm_component_tasks *>(g + stride * r + L.comps)[c];
      t.started += x.started;
      t.finished += x.finished;
    }
    t.in_flight = t.started - t.finished;
    p.comps[c] = t;
  }
  for (size_t b = tid; b < p.nb; b += nth) {
    rtm_buffer_stat pick = reinterpret_cast<const rtm_buffer_stat *>(g + L.bstat)[b];
    for (unsigned r = 0; r < world; ++r) {
      const rtm_buffer_stat x = reinterpret_cast<const rtm_buffer_stat *>(g + stride * r + L.bstat)[b];
      if (x.reserved) { pick = x; break; }
    }
    p.bstat[b] = pick;
  }
}

}  // namespace

// ============================================================================================
// launchers
// ============================================================================================
size_t fold_smem_bytes() { return sizeof(FoldSmem) * kFoldWarps; }
size_t partition_smem_bytes(uint32_t nbins) {
  return (size_t)kTileS * 8 + (size_t)(nbins + 1) * 4 + (size_t)8 * nbins * 2 + 16;
}
size_t topk_smem_bytes(uint32_t nb) {
  return (size_t)(nb <= kTopkSmemKeys ? ((nb + 1) & ~1u) : 0) * 4 + 16 * 256 * 4 + 1024 * 8;
}

void launch_split(const Params &p, bool samples, long long *outB, cudaStream_t st) {
  const unsigned warps = p.W + 1;
  const unsigned threads = 128;
  const unsigned blocks = (warps * 32 + threads - 1) / threads;
  if (samples) k_split<true><<<blocks, threads, 0, st>>>(p, outB);
  else k_split<false><<<blocks, threads, 0, st>>>(p, outB);
}

void launch_fill_tile_regions(const Params &p, cudaStream_t st) {
  const unsigned nr = p.W + 2;
  const unsigned blocks = nr < 4096 ? nr : 4096;
  if (p.n_tiles_s) k_fill_tile_regions<<<blocks, 64, 0, st>>>(p.rts, const_cast<uint32_t *>(p.tile_reg_s), nr);
  if (p.n_tiles_e) k_fill_tile_regions<<<blocks, 64, 0, st>>>(p.rte, const_cast<uint32_t *>(p.tile_reg_e), nr);
}

void launch_partition(const Params &p, cudaStream_t st) {
  if (!p.n_tiles_s) return;
  const size_t sm = partition_smem_bytes(p.nbins);
  k_partition<<<p.n_tiles_s, kK1Threads, sm, st>>>(p);
}

void launch_events(const Params &p, cudaStream_t st) {
  if (!p.n_tiles_e) return;
  const size_t sm = (size_t)2 * p.nk * 4 + (p.ncw <= 2048 ? (size_t)p.ncw * 4 : 0);
  k_events<<<p.n_tiles_e, kK3Threads, sm, st>>>(p);
}

void launch_fold(const Params &p, int n_sms, cudaStream_t st) {
  const size_t sm = fold_smem_bytes();
  int per_sm = 0;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_fold, kFoldWarps * 32, sm);
  if (per_sm < 1) per_sm = 1;
  unsigned grid = (unsigned)(n_sms * per_sm);
  const unsigned units = p.W * p.nbins;
  const unsigned need = (units + kFoldWarps - 1) / kFoldWarps;
  if (grid > need) grid = need;
  if (grid == 0) grid = 1;
  k_fold<<<grid, kFoldWarps * 32, sm, st>>>(p);
}

void launch_order_check(const Params &p, cudaStream_t st) {
  if (p.n_tiles_s) k_order_check<<<1, 1024, 0, st>>>(p.smeta, p.n_tiles_s, p.status, 1u);
  if (p.n_tiles_e) k_order_check<<<1, 1024, 0, st>>>(p.emeta, p.n_tiles_e, p.status, 2u);
}

void launch_topk(const Params &p, cudaStream_t st) {
  k_topk<<<p.W, kTopkThreads, topk_smem_bytes(p.nb), st>>>(p);
}

void launch_hang(const Params &p, cudaStream_t st) {
  const unsigned threads = 128;
  const unsigned blocks = (p.ncw * 32 + threads - 1) / threads;
  k_hang<<<blocks, threads, 0, st>>>(p);
}

void launch_progress(const Params &p, cudaStream_t st) {
  const unsigned comp_blocks = (p.nc + 255) / 256 < 256 ? (p.nc + 255) / 256 : 256;
  k_progress<<<p.nk + comp_blocks, 256, 0, st>>>(p);
}

uint64_t pack_bytes(const Params &p) { return pack_layout(p).total; }

void configure_kernels_once() {
  static bool done[128] = {false};
  int dev = 0;
  cudaGetDevice(&dev);
  if (dev < 0 || dev >= 128 || done[dev]) return;
  done[dev] = true;
  cudaFuncSetAttribute(k_partition, cudaFuncAttributeMaxDynamicSharedMemorySize,
                       (int)partition_smem_bytes(kMaxBins));
  cudaFuncSetAttribute(k_topk, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)topk_smem_bytes(kTopkSmemKeys));
  cudaFuncSetAttribute(k_fold, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)fold_smem_bytes());
  cudaGetLastError();
}

void launch_pack(const Params &p, void *pack, cudaStream_t st) {
  const PackLayout L = pack_layout(p);
  unsigned char *d = static_cast<unsigned char *>(pack);
  cudaMemcpyAsync(d + L.win, p.win, (size_t)kWinFields * p.W * 8, cudaMemcpyDeviceToDevice, st);
  cudaMemcpyAsync(d + L.topk, p.topk, (size_t)p.W * p.k * 8, cudaMemcpyDeviceToDevice, st);
  cudaMemcpyAsync(d + L.topk_n, p.topk_n, (size_t)p.W * 4, cudaMemcpyDeviceToDevice, st);
  cudaMemcpyAsync(d + L.prog, p.prog, (size_t)p.W * p.nk * 5 * 8, cudaMemcpyDeviceToDevice, st);
  cudaMemcpyAsync(d + L.hung, p.hung, (size_t)p.W * p.ncw * 4, cudaMemcpyDeviceToDevice, st);
  cudaMemcpyAsync(d + L.comps, p.comps, (size_t)p.nc * sizeof(rtm_component_tasks), cudaMemcpyDeviceToDevice, st);
  cudaMemcpyAsync(d + L.bstat, p.bstat, (size_t)p.nb * sizeof(rtm_buffer_stat), cudaMemcpyDeviceToDevice, st);
}

void launch_merge(const Params &p, const void *gathered, uint32_t world, cudaStream_t st) {
  const size_t stride = pack_layout(p).total;
  unsigned P = 1;
  while (P < world * p.k) P <<= 1;
  const size_t sm = (size_t)P * 16;
  if (sm > 48 * 1024) cudaFuncSetAttribute(k_merge_windows, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
  k_merge_windows<<<p.W, 256, sm, st>>>(p, static_cast<const unsigned char *>(gathered), world, stride);
  k_merge_tables<<<256, 256, 0, st>>>(p, static_cast<const unsigned char *>(gathered), world, stride);
}

}  // namespace rtm
