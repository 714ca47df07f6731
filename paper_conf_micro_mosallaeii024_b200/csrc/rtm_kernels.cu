// rtm_kernels.cu — sm_100a kernels of the window-snapshot reduction (see rtm_internal.h and
// DESIGN.md §4).  No tensor cores: nothing here is a dense contraction; the path is bound by
// the one compulsory HBM read of 16 B per trace record.
#include <cooperative_groups.h>
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdlib.h>

#include <type_traits>

#include <algorithm>
#include <atomic>
#include <map>
#include <mutex>
#include <tuple>

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
__device__ __forceinline__ unsigned ld_relaxed_u32(const unsigned *p) {
  unsigned v;
  asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
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

// Lanes holding the same BITS-bit key: one ballot per key bit.  On sm_100 __match_any_sync costs
// ~59 cycles of SM throughput per warp instruction; this costs ~2.5 per bit (tools/microbench.cu).
template <int BITS>
__device__ __forceinline__ unsigned match_bits(unsigned key) {
  unsigned m = kFull;
#pragma unroll
  for (int k = 0; k < BITS; ++k) {
    // m &= bit_k(key) ? ballot : ~ballot   -- predicate, VOTE, two predicated LOP3s
    asm("{\n .reg .pred p;\n .reg .b32 b;\n"
        " setp.ne.u32 p, %1, 0;\n"
        " vote.sync.ballot.b32 b, p, 0xffffffff;\n"
        " @p  and.b32 %0, %0, b;\n"
        " not.b32 b, b;\n"
        " @!p and.b32 %0, %0, b;\n}"
        : "+r"(m)
        : "r"(key & (1u << k)));
  }
  return m;
}

// field validity (include/rtm.h)
__device__ __forceinline__ bool sample_valid(const Params &p, const int4 &v) {
  unsigned b = (unsigned)v.z, lvl = (unsigned)v.w & 0xFFFFu, c = (unsigned)v.w >> 16;
  return b < p.nb && c == (unsigned)__ldg(p.cap + b) && lvl <= c;
}
__device__ __forceinline__ bool event_valid(const Params &p, const int4 &v) {
  unsigned meta = (unsigned)v.w;
  const unsigned kern = (meta >> 20) & 0x7FFu;
  return (meta & 0xFFFFFu) < p.nc && kern < p.nk && (p.all_live || __ldg(p.klive + kern));
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
__device__ __forceinline__ void split_one(const Params &p, unsigned q, long long *outB) {
  const int lane = threadIdx.x & 31;
  const long long T = p.t_inline ? p.Tin[q] : p.T[q];
  const unsigned long long N = SAMPLES ? p.ns : p.ne;
  const int4 *recs = SAMPLES ? reinterpret_cast<const int4 *>(p.s) : reinterpret_cast<const int4 *>(p.e);
  unsigned long long lo = 0, hi = N;
  // Fast exits for the call's outer boundaries (one probe round instead of the search; the
  // common streaming call ingests exactly its windows' records): the first boundary is 0 when the
  // stream's first field-valid record is at or after it, the last is 1 + the index of the last
  // field-valid record when that one is before it (sorted stream; an unsorted one is reported by
  // the order check).
  if ((q == 0 || q == p.W) && N > 0) {
    const bool first = q == 0;
    const unsigned long long i = first ? (unsigned long long)lane : N - 1 - (unsigned long long)lane;
    bool ok = false;
    long long ts = 0;
    if (i < N) {
      const int4 v = __ldcg(recs + i);
      ok = SAMPLES ? sample_valid(p, v) : event_valid(p, v);
      ts = rec_ts(v);
    }
    const unsigned m = __ballot_sync(kFull, ok);
    if (m) {
      const int src = __ffs(m) - 1;  // first: lowest index; last: lane 0 probes N - 1
      const long long t = __shfl_sync(kFull, ts, src);
      if (first ? t >= T : t < T) {
        if (lane == 0) outB[q] = first ? 0 : (long long)(N - (unsigned long long)src);
        return;
      }
    }
  }
  while (hi - lo > 64) {  // then <= 2 dependent rounds of the final scan
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


// Region boundaries -> tile table on the device (no host round trip): B[0] = 0, B[W+2] = N, the
// split positions made monotone (only an unsorted stream can break that; it is reported by the
// order check), rt[r] = first tile of region r, rt[W+2] = number of tiles.  One CTA.
__device__ __forceinline__ void regions_one(long long *B, unsigned long long N, uint32_t W, uint32_t *rt, int tile) {
  __shared__ long long wmax[32];
  __shared__ unsigned wsum[32];
  __shared__ long long carry_m;
  __shared__ unsigned carry_s;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const unsigned nr = W + 3;
  if (threadIdx.x == 0) { carry_m = 0; carry_s = 0; }
  __syncthreads();
  for (unsigned base = 0; base < nr; base += blockDim.x) {  // prefix max of the positions
    const unsigned r = base + threadIdx.x;
    long long x = 0;
    if (r < nr) x = r == 0 ? 0 : (r == nr - 1 ? (long long)N : B[r]);
    if (x > (long long)N) x = (long long)N;
    for (int o = 1; o < 32; o <<= 1) {
      const long long y = __shfl_up_sync(kFull, x, o);
      if (lane >= o && y > x) x = y;
    }
    if (lane == 31) wmax[warp] = x;
    __syncthreads();
    long long pre = carry_m;
    for (int w = 0; w < warp; ++w) pre = wmax[w] > pre ? wmax[w] : pre;
    if (pre > x) x = pre;
    __syncthreads();
    if (r < nr) B[r] = x;
    if (threadIdx.x == blockDim.x - 1) carry_m = x;
    __syncthreads();
  }
  for (unsigned base = 0; base < nr; base += blockDim.x) {  // tiles per region, exclusive sum
    const unsigned r = base + threadIdx.x;
    unsigned cnt = 0;
    if (r + 1 < nr) cnt = (unsigned)((B[r + 1] - B[r] + tile - 1) / tile);
    unsigned x = cnt;
    for (int o = 1; o < 32; o <<= 1) {
      const unsigned y = __shfl_up_sync(kFull, x, o);
      if (lane >= o) x += y;
    }
    if (lane == 31) wsum[warp] = x;
    __syncthreads();
    unsigned pre = carry_s;
    for (int w = 0; w < warp; ++w) pre += wsum[w];
    __syncthreads();
    if (r < nr) rt[r] = pre + x - cnt;
    if (threadIdx.x == blockDim.x - 1) carry_s = pre + x;
    __syncthreads();
  }
}

// tile tables of region r: the sample tiles' region id + descriptor (start, bounds, size, window)
// and the event tiles' region id
__device__ __forceinline__ void fill_region(const Params &p, uint32_t r, bool samples, bool events) {
  if (events)
    for (uint32_t t = p.rte[r] + threadIdx.x; t < p.rte[r + 1]; t += blockDim.x)
      const_cast<uint32_t *>(p.tile_reg_e)[t] = r;
  if (!samples) return;
  const Region g = region_of(p, r);
  const long long lo = g.lo_ts;
  const unsigned long long wlen =
      g.hi_ts == kTsMax ? (unsigned long long)(kTsMax - lo) + 1ull : (unsigned long long)(g.hi_ts - lo);
  for (uint32_t t = p.rts[r] + threadIdx.x; t < p.rts[r + 1]; t += blockDim.x) {
    const_cast<uint32_t *>(p.tile_reg_s)[t] = r;
    TileDesc d;
    d.start = p.Bs[r] + (long long)(t - p.rts[r]) * kTileS;
    long long endp = p.Bs[r + 1];
    if (endp > d.start + kTileS) endp = d.start + kTileS;
    d.n = (int)(endp - d.start);
    d.lo = lo;
    d.wlen = wlen;
    d.window = g.window;
    d.charge = g.charge;
    d.pad[0] = d.pad[1] = d.pad[2] = 0;
    p.tdesc[t] = d;
  }
}

// zero every range of the list: 16-byte stores over each range's 16-byte-aligned body, bytes
// for the ends (ranges come from cudaMalloc'd buffers and may have any length)
__device__ __forceinline__ void clear_ranges(const ClearList &cl) {
  const size_t tid = (size_t)blockIdx.x * blockDim.x + threadIdx.x, nth = (size_t)gridDim.x * blockDim.x;
  for (int r = 0; r < cl.n; ++r) {
    unsigned char *b = static_cast<unsigned char *>(cl.ptr[r]);
    const size_t n = cl.bytes[r];
    const size_t head = (16 - ((uintptr_t)b & 15)) & 15;
    const size_t h = head < n ? head : n;
    const size_t body = (n - h) / 16;
    if (tid < h) b[tid] = 0;
    uint4 *b4 = reinterpret_cast<uint4 *>(b + h);
    for (size_t i = tid; i < body; i += nth) b4[i] = make_uint4(0, 0, 0, 0);
    for (size_t i = h + body * 16 + tid; i < n; i += nth) b[i] = 0;
  }
}

// The prologue of a reduce call in ONE cooperative launch (it was four: clear, split, regions,
// tile tables): (A) zero the call's accumulators and find the region boundaries (one warp per
// window boundary and stream), grid barrier, (B) boundaries -> per-region tile counts (blocks 0 and
// 1), grid barrier, (C) the tile tables.  Every phase is grid-strided, so any co-resident grid works.
#ifndef RTM_TU_PARTITION
__global__ void __launch_bounds__(256, 4) k_prep(Params p, ClearList cl, long long *Bs, long long *Be) {
  namespace cg = cooperative_groups;
  cg::grid_group grid = cg::this_grid();
  if (p.t_inline && blockIdx.x == 0 && threadIdx.x <= p.W) const_cast<long long *>(p.T)[threadIdx.x] = p.Tin[threadIdx.x];
  clear_ranges(cl);
  const unsigned nwarps = gridDim.x * (blockDim.x >> 5);
  for (unsigned q = (blockIdx.x * blockDim.x + threadIdx.x) >> 5; q <= 2 * p.W + 1; q += nwarps) {
    if (q <= p.W) split_one<true>(p, q, Bs + 1);
    else split_one<false>(p, q - (p.W + 1), Be + 1);
  }
  // a one-block grid (few-window calls) synchronises with a block barrier
  auto gsync = [&]() {
    if (gridDim.x == 1) __syncthreads();
    else grid.sync();
  };
  gsync();
  if (blockIdx.x == 0) regions_one(Bs, p.ns, p.W, const_cast<uint32_t *>(p.rts), kTileS);
  if (blockIdx.x == (gridDim.x > 1 ? 1u : 0u)) regions_one(Be, p.ne, p.W, const_cast<uint32_t *>(p.rte), kTileE);
  gsync();
  for (uint32_t r = blockIdx.x; r < p.W + 2; r += gridDim.x) fill_region(p, r, true, true);
}
#endif

// ============================================================================================
// K3: task events.  One CTA per tile of <= 4096 events of one region: validate, order-check,
// per-(window, kernel) START/END counts, per-(window, component) activity bits and per-call
// per-component START/END deltas (progress bars, L131; "task counts stop changing", L227).
// ============================================================================================
// One event tile, by a whole CTA of kK3Threads (also run inside the persistent partition kernel,
// after its sample tiles: smem = the CTA's dynamic shared memory, >= events_smem_bytes).
__device__ __forceinline__ void events_tile(const Params &p, unsigned tile, unsigned char *smem) {
  unsigned *khist = reinterpret_cast<unsigned *>(smem);  // [nk*2]
  unsigned *abits = khist + 2 * p.nk;                     // [ncw] if smem_bits
  __shared__ long long wfirst[8], wlast[8];
  __shared__ unsigned whas[8], wviol[8], wkept[8];
  const bool smem_bits = p.ncw <= 2048;

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
        atomicAdd(p.cdelta + 2 * comp + kind, 1ull);  // one RED per event: measured cheaper than aggregating
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
  if (is_win) {
    for (unsigned i = threadIdx.x; i < 2 * p.nk; i += blockDim.x)
      if (khist[i]) atomicAdd(p.kdelta + ((size_t)g.window * p.nk) * 2 + i, khist[i]);
    if (smem_bits)
      for (unsigned i = threadIdx.x; i < p.ncw; i += blockDim.x)
        if (abits[i]) atomicOr(p.active + (size_t)g.window * p.ncw + i, abits[i]);
  }
  __syncthreads();  // shared memory free for the next tile
}

#ifndef RTM_TU_PARTITION
__global__ void __launch_bounds__(kK3Threads) k_events(Params p) {
  if (blockIdx.x >= p.rte[p.W + 2]) return;  // grid sized by an upper bound
  extern __shared__ __align__(16) unsigned char smem[];
  events_tile(p, blockIdx.x, smem);
}
#endif

// ============================================================================================
// K1: sample partition.  A tile is <= 4096 samples of ONE region, handled by one CTA of 8 warps;
// warp w owns the sub-tile [512w, 512w + 512).  Per sample: field validity, range + order check
// against the previous field-valid sample, and a stable multisplit by bin (buffer_id >> 8).  Kept
// samples become 8-byte entries  (ts - t_begin) << 24 | level << 8 | (buffer_id & 255).
//
// k_partition_lm (lane-major, n_bins <= 128; persistent, 1-2 CTAs per SM): the buffer-capacity
// table lives in shared memory (the field check is a gather per sample: from L1 it was the
// kernel's bottleneck).  Each warp stages its 512 raw records in shared memory (XOR-swizzled
// 16-byte slots) and lane l takes the CONSECUTIVE records 16l .. 16l+15, so the stable order
// inside a bin is (lane, slot).  No warp collectives: rank = a u8 (bin, lane) counter in the
// warp's (consumed) raw slot; each lane then prefix-scans whole bin rows with byte-SIMD
// multiplies, so position = rank + earlier lanes' counts of the bin.
// k_partition_mx (fallback, any n_bins): lanes take strided records; __match_any_sync peers +
// the warp's bin counters give the rank.
//
// Both: one barrier publishes every warp's bin totals; each warp derives its bin bases (CTA bin
// offsets + earlier warps' counts) and permutes its entries into a CTA buffer that reuses the raw
// staging; a second barrier precedes the coalesced copy-out.  soff gets the tile's u16 bin offsets.
// ============================================================================================
constexpr int kSub = kTileS / (kK1Threads / 32);  // 512 samples per warp
constexpr int kPerLane = kSub / 32;               // 16
constexpr int kK1Warps = kK1Threads / 32;         // 8
constexpr unsigned kNoKey = 0xFFFFu;
static_assert(kPerLane == 16, "lane-major swizzle assumes 16 records per lane");
static_assert((size_t)kLmMaxBins * 48 <= (size_t)kSub * 16, "count rows must fit the raw slot");

struct K1WarpSum {
  unsigned long long first, last;  // offsets of the first / last field-valid record
  unsigned has, viol, kept, pad;
};

__host__ __device__ constexpr size_t k1_align16(size_t x) { return (x + 15) & ~(size_t)15; }
__host__ __device__ constexpr size_t k1_vec_bytes(uint32_t nbins) { return k1_align16((size_t)kK1Warps * nbins * 2); }
// dynamic shared memory.  lm: raw 16 B x 4096 | wt x 2 (tile parity) | wb | tile descriptors
// (8 warps x 2) | cap[nb];  mx: sbuf 8 B x 4096 | wt | wb
// (wt: 8 x nbins u16 bin totals / live counters, wb: 8 x nbins u16 bin bases)
__host__ __device__ constexpr size_t k1_smem_lm(uint32_t nbins, uint32_t nb, bool caps = true) {
  return (size_t)kTileS * 16 + 3 * k1_vec_bytes(nbins) + (size_t)kK1Warps * 2 * sizeof(TileDesc) +
         (caps ? k1_align16((size_t)nb * 2) : 0);
}
__host__ __device__ constexpr size_t k1_smem_mx(uint32_t nbins) { return (size_t)kTileS * 8 + 2 * k1_vec_bytes(nbins); }

#ifdef RTM_TU_PARTITION  // the partition kernels: compiled in their own module (rtm_partition.cu)
struct K1Tile {
  unsigned tile;
  int n;
  Region g;
  long long lo;
  unsigned long long wlen;
  long long start;
};
__device__ __forceinline__ K1Tile k1_tile_from(const TileDesc &d, unsigned tile) {
  K1Tile t;
  t.tile = tile;
  t.start = d.start;
  t.n = d.n;
  t.g.lo_ts = d.lo;
  t.g.hi_ts = 0;  // unused: the bound is (lo, wlen)
  t.g.window = d.window;
  t.g.charge = d.charge;
  t.lo = d.lo;
  t.wlen = d.wlen;
  return t;
}
__device__ __forceinline__ K1Tile k1_tile(const Params &p, unsigned tile) { return k1_tile_from(p.tdesc[tile], tile); }

__device__ __forceinline__ void cp_async16(void *smem_dst, const void *gsrc) {
  const unsigned d = (unsigned)__cvta_generic_to_shared(smem_dst);
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;\n" ::"r"(d), "l"(gsrc) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;\n" ::: "memory"); }
__device__ __forceinline__ void cp_async_wait_all() { asm volatile("cp.async.wait_all;\n" ::: "memory"); }
__device__ __forceinline__ void cp_async_wait_1() { asm volatile("cp.async.wait_group 1;\n" ::: "memory"); }

// After B1: tile meta + drop / kept counts (warp 0), in warp order.
__device__ __forceinline__ void k1_tile_summary(const Params &p, const K1Tile &t, const K1WarpSum *wsum) {
  const int lane = threadIdx.x & 31;
  K1WarpSum x;
  x.first = x.last = 0;
  x.has = x.viol = x.kept = x.pad = 0;
  if (lane < kK1Warps) x = wsum[lane];
  const unsigned hm = __ballot_sync(kFull, x.has != 0);
  const unsigned lower = hm & lanemask_lt();
  const unsigned long long pl = __shfl_sync(kFull, x.last, lower ? 31 - __clz(lower) : lane);
  const bool bad = (x.viol != 0) | ((x.has != 0) & (lower != 0) & (x.first < pl));
  const bool tv = __any_sync(kFull, bad);
  const unsigned tk = warp_sum(x.kept);
  const unsigned long long tf = __shfl_sync(kFull, x.first, hm ? __ffs(hm) - 1 : 0);
  const unsigned long long tl = __shfl_sync(kFull, x.last, hm ? 31 - __clz(hm) : 0);
  if (lane == 0) {
    TileMeta m;
    m.first_ts = (long long)((unsigned long long)t.lo + tf);
    m.last_ts = (long long)((unsigned long long)t.lo + tl);
    m.flags = (hm ? 1u : 0u) | (tv ? 2u : 0u);
    m.pad = 0;
    p.smeta[t.tile] = m;
    if ((unsigned)t.n > tk) atomicAdd(p.win + WF_DROPPED * p.W + t.g.charge, (unsigned long long)(t.n - tk));
    if (tk) atomicAdd(p.win + WF_SAMPLES * p.W + t.g.window, (unsigned long long)tk);
  }
}

// After B1 (window tiles): this warp's bin bases -> myb; warp 0 writes the soff row.  Returns the
// tile's kept total.
template <int KS>
__device__ __forceinline__ unsigned k1_bin_bases(const Params &p, unsigned tile, const unsigned short *wt,
                                                 unsigned short *myb) {
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const unsigned nbins = KS == kSupLog ? p.nsb : p.nbins;
  uint16_t *offs = p.soff + (size_t)tile * (nbins + 1);
  unsigned carry = 0;
  for (unsigned b0 = 0; b0 < nbins; b0 += 32) {
    const unsigned b = b0 + lane;
    unsigned T = 0, P = 0;
    if (b < nbins) {
#pragma unroll
      for (int w2 = 0; w2 < kK1Warps; ++w2) {
        const unsigned x = wt[(size_t)w2 * nbins + b];
        T += x;
        P += w2 < warp ? x : 0u;
      }
    }
    unsigned incl = T;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const unsigned y = __shfl_up_sync(kFull, incl, o);
      if (lane >= o) incl += y;
    }
    const unsigned base = carry + incl - T;
    if (b < nbins) {
      myb[b] = (unsigned short)(base + P);
      if (warp == 0) offs[b] = (uint16_t)base;
    }
    carry += __shfl_sync(kFull, incl, 31);
  }
  if (warp == 0 && lane == 0) offs[nbins] = (uint16_t)carry;
  __syncwarp();
  return carry;
}

__device__ __forceinline__ void k1_publish(K1WarpSum *wsum, unsigned long long first, unsigned long long last,
                                           bool has, bool viol, unsigned kept) {
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  kept = warp_sum(kept);
  viol = __any_sync(kFull, viol);
  if (lane == 0) {
    K1WarpSum s;
    s.first = first;
    s.last = last;
    s.has = has;
    s.viol = viol;
    s.kept = kept;
    s.pad = 0;
    wsum[warp] = s;
  }
}

// One lane's 16 consecutive records: field check, running min / max of the field-valid offsets
// (an inversion inside the lane shows up as an offset below the running max), entries, keys.
// NAR: windows shorter than 2^32 ticks, so offsets are compared and packed in 32 bits.
// KS: key = buffer_id >> KS.  KS == 8: the 256-buffer bin (entries as above); KS == 7: the
// 128-buffer bin (entries off << 23 | level << 7 | buffer_id & 127: few-unit calls, see rtm_api.cpp);
// KS == kSupLog: the superbin of the two-pass path (narrow windows only): entry =
// o << 32 | level << 16 | (buffer_id & 0x3FFF).
template <bool NAR, int BL, bool CAPS, int KS>
__device__ __forceinline__ void lm_scan(const Params &p, const K1Tile &t, bool is_win, const int4 *raw,
                                        const unsigned short *capS, int sub0, unsigned long long (&e)[kPerLane],
                                        unsigned (&kp)[kPerLane], unsigned long long &first,
                                        unsigned long long &last, bool &has, bool &viol, unsigned &kept) {
  const int lane = threadIdx.x & 31;
  unsigned mn = ~0u, mx = 0u, hiacc = 0u;
  unsigned long long mn64 = ~0ull, mx64 = 0ull;
  bool hv = false, bad = false;
#pragma unroll
  for (int k = 0; k < kPerLane; ++k) {
    const int i = lane * kPerLane + k;
    const int4 v = raw[lane * kPerLane + (k ^ (lane & 7))];
    const unsigned b = (unsigned)v.z, lvl = (unsigned)v.w & 0xFFFFu, c = (unsigned)v.w >> 16;
    const unsigned capb = CAPS ? capS[b < p.nb ? b : 0u] : (unsigned)__ldg(p.cap + (b < p.nb ? b : 0u));
    const bool valid = (sub0 + i < t.n) & (b < p.nb) & (c == capb) & (lvl <= c);
    const unsigned long long off = (unsigned long long)(rec_ts(v) - t.lo);
    hv |= valid;
    if (NAR) {
      const unsigned o = (unsigned)off;
      bad |= valid & (o < mx);
      mx = max(mx, valid ? o : 0u);
      mn = min(mn, valid ? o : ~0u);
      hiacc |= valid ? (unsigned)(off >> 32) : 0u;
      if constexpr (KS == kSupLog) {
        e[k] = ((unsigned long long)o << 32) | (lvl << 16) | (b & ((1u << kSupLog) - 1u));
      } else if constexpr (KS != 8) {
        e[k] = ((unsigned long long)o << (16 + KS)) | (lvl << KS) | (b & ((1u << KS) - 1u));
      } else {
        // (o << 24) | (level << 8) | (buffer_id & 255), o < 2^32
        const unsigned lo = __byte_perm(__byte_perm((unsigned)v.z, (unsigned)v.w, 0x0540), o, 0x4210);
        e[k] = ((unsigned long long)(o >> 8) << 32) | lo;
      }
    } else {
      bad |= valid & (off < mx64);
      mx64 = max(mx64, valid ? off : 0ull);
      mn64 = min(mn64, valid ? off : ~0ull);
      constexpr int EB = KS == kSupLog ? BL : KS;  // bin bits of a fold entry
      e[k] = (off << (16 + EB)) | ((unsigned long long)lvl << EB) | (b & ((1u << EB) - 1u));
    }
    const bool keep = valid & is_win;
    kept += keep;
    kp[k] = (keep ? (b >> KS) : kNoKey) << 16;
  }
  if (NAR) {
    bad |= hv & ((hiacc != 0u) | ((unsigned long long)mx >= t.wlen));
    first = mn;
    last = mx;
  } else {
    bad |= hv & (mx64 >= t.wlen);
    first = mn64;
    last = mx64;
  }
  has = hv;
  viol = bad;
}

#ifdef RTM_PHASE_TIMING
// thread 0's view of a persistent kernel's per-tile phases (cycles), summed into p.dbg[slot]
#define PTM(slot_)                                                       \
  do {                                                                   \
    if (threadIdx.x == 0 && p.dbg) {                                     \
      const long long t1_ = clock64();                                   \
      atomicAdd(p.dbg + (slot_), (unsigned long long)(t1_ - pt_));       \
      pt_ = t1_;                                                         \
    }                                                                    \
  } while (0)
#else
#define PTM(slot_) \
  do {             \
  } while (0)
#endif

// After the tile's barrier the warps permute their entries into the first half of the raw staging
// (shared memory), a second barrier, then warps 0-3 copy the tile out with coalesced 16-byte stores
// and only then prefetch their next raw records (named barrier among themselves); warps 4-7
// prefetch before the first barrier (measured 813 -> 692 us on C2 against direct 8-byte scatter
// stores from every lane, which touched 32 sectors per store instruction).
template <int BL, bool CAPS, int KS, bool MP>
__global__ void __launch_bounds__(kK1Threads, 2) k_partition_lm(Params p) {
  static_assert(BL == 8, "lane-major entries pack the buffer id in one byte");
  static_assert(!MP || KS != kSupLog, "multi-pass ranking: bins");
  static_assert(KS == 8 || KS == 7 || KS == kSupLog, "bins or superbins");
  extern __shared__ __align__(16) unsigned char smem[];
  __shared__ K1WarpSum wsum[2][kK1Warps];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const unsigned lt = lanemask_lt();
  const unsigned nbins = KS == kSupLog ? p.nsb : p.nbins;
  const size_t vb = k1_vec_bytes(nbins);
  unsigned char *tail = smem + (size_t)kTileS * 16;
  unsigned short *wt2 = reinterpret_cast<unsigned short *>(tail);            // [2][8][nbins]
  unsigned short *myb = reinterpret_cast<unsigned short *>(tail + 2 * vb) + (size_t)warp * nbins;
  TileDesc *dsm = reinterpret_cast<TileDesc *>(tail + 3 * vb) + warp * 2;     // this warp's [2]
  unsigned short *capS = reinterpret_cast<unsigned short *>(tail + 3 * vb + (size_t)kK1Warps * 2 * sizeof(TileDesc));
  int4 *raw = reinterpret_cast<int4 *>(smem) + warp * kSub;  // this warp's slot
  // after the scan the slot holds the count rows: 48 B per bin = 32 u8 lane counters (later the
  // exclusive in-word prefixes) + 8 u16 word bases
  unsigned char *rows = reinterpret_cast<unsigned char *>(raw);
  if (CAPS)  // the capacity table in shared memory (the field check gathers it per sample)
  {  // 16-byte loads (8 capacities each): this fill is on the critical path of one-window calls
    const unsigned n8 = p.nb >> 3;
    const uint4 *src = reinterpret_cast<const uint4 *>(p.cap);
    uint4 *dst = reinterpret_cast<uint4 *>(capS);
    for (unsigned i = threadIdx.x; i < n8; i += kK1Threads) dst[i] = __ldg(src + i);
    for (unsigned i = (n8 << 3) + threadIdx.x; i < p.nb; i += kK1Threads) capS[i] = __ldg(p.cap + i);
  }
  // Tiles are claimed dynamically (p.unit_ctr[1]) so a CTA that starts late - the side-stream
  // event kernel holds SMs at first - simply takes fewer tiles.  Claims run two ahead:
  // ring[i & 3] is iteration i's tile, written by thread 0 in iteration i - 2 and read after
  // the barrier of iteration i - 1.
  __shared__ unsigned ring[4];
  const unsigned n_tiles = p.rts[p.W + 2];
  auto claim = [&]() -> unsigned {
    const unsigned t = atomicAdd(p.unit_ctr + 1, 1u);
    return t < n_tiles ? t : ~0u;
  };
  if (threadIdx.x == 0) {
    ring[0] = claim();
    ring[1] = ring[0] != ~0u ? claim() : ~0u;
  }
  const int sub0 = warp * kSub;
  // async prefetch of a tile (descriptor already in dsm[slot]): this warp's 512 raw records,
  // record i to the 16-byte slot 16(i>>4) + ((i&15) ^ ((i>>4)&7))
  auto prefetch_raw = [&](const TileDesc &d) {
    const int4 *src = reinterpret_cast<const int4 *>(p.s) + d.start + sub0;
    const int m = d.n - sub0;
#pragma unroll
    for (int j = 0; j < kPerLane; ++j) {
      const int i = j * 32 + lane;
      if (i < m) cp_async16(raw + ((i & ~15) | ((i & 15) ^ ((i >> 4) & 7))), src + i);
    }
  };
  __syncthreads();  // capacity table, ring[0..1]
  unsigned tile = ring[0];
  if (tile != ~0u) {
    if (lane < 3) cp_async16(reinterpret_cast<int4 *>(dsm) + lane, reinterpret_cast<const int4 *>(p.tdesc + tile) + lane);
    cp_async_commit();
    cp_async_wait_all();
    __syncwarp();
    prefetch_raw(dsm[0]);
  }
  cp_async_commit();
  long long pt_ = clock64();
  (void)pt_;
  for (unsigned it = 0, par = 0; tile != ~0u; ++it, par ^= 1) {
    const unsigned nxt = ring[(it + 1) & 3];
    if (threadIdx.x == 0) ring[(it + 2) & 3] = nxt != ~0u ? claim() : ~0u;
    const K1Tile t = k1_tile_from(dsm[par], tile);
    const bool is_win = t.g.window >= 0;
    unsigned short *wt = wt2 + (size_t)par * (vb / 2);
    unsigned short *myt = wt + (size_t)warp * nbins;
    __syncwarp();  // dsm[par] read by every lane before it is reused
    if (nxt != ~0u && lane < 3)
      cp_async16(reinterpret_cast<int4 *>(dsm + (par ^ 1)) + lane, reinterpret_cast<const int4 *>(p.tdesc + nxt) + lane);
    cp_async_commit();
    cp_async_wait_1();  // this tile's raw records (the descriptor group may still be in flight)
    __syncwarp();
    PTM(1);
    if (threadIdx.x == 0 && p.dbg) atomicAdd(p.dbg + 7, 1ull);
    unsigned long long e[kPerLane];
    unsigned kp[kPerLane];  // key << 16 | position within the warp's bin group
    unsigned long long first, last;
    bool has, viol;
    unsigned kept = 0;
    if (p.narrow && is_win) lm_scan<true, BL, CAPS, KS>(p, t, is_win, raw, capS, sub0, e, kp, first, last, has, viol, kept);
    else lm_scan<false, BL, CAPS, KS>(p, t, is_win, raw, capS, sub0, e, kp, first, last, has, viol, kept);
    {  // order across lanes: my first vs the last of the nearest earlier lane with a valid record
      const unsigned hm = __ballot_sync(kFull, has);
      const unsigned lower = hm & lt;
      const unsigned long long pl = __shfl_sync(kFull, last, lower ? 31 - __clz(lower) : lane);
      viol |= has & (lower != 0) & (first < pl);
      const unsigned long long f0 = __shfl_sync(kFull, first, hm ? __ffs(hm) - 1 : 0);
      const unsigned long long l0 = __shfl_sync(kFull, last, hm ? 31 - __clz(hm) : 0);
      first = f0;
      last = l0;
      has = hm != 0;
    }
    PTM(2);
    __syncwarp();  // every lane has consumed its raw records
    if (is_win) {  // rank = (lane, bin) counter; position = rank + earlier lanes' counts of the bin
      // bins [kb, kb + nk): their count rows (48 B per bin) overlay the consumed raw slot.  MP
      // (171 .. 1023 bins): the slot holds the rows of at most kLmMaxBins bins, so the keys are
      // ranked in passes over bin ranges (each record in the pass of its bin).
      if constexpr (MP) {
        auto rank_pass = [&](unsigned kb, unsigned nk) {
          uint4 *r4 = reinterpret_cast<uint4 *>(rows);
          for (unsigned q = lane; q < nk * 3; q += 32) r4[q] = make_uint4(0, 0, 0, 0);
          __syncwarp();
  #pragma unroll
          for (int k = 0; k < kPerLane; ++k) {
            const unsigned key = kp[k] >> 16, rk = key - kb;
            if (key != kNoKey && (!MP || rk < nk)) {
              unsigned char *ctr = rows + rk * 48 + lane;
              const unsigned r = *ctr;
              *ctr = (unsigned char)(r + 1);
              kp[k] |= r;
            }
          }
          __syncwarp();
          for (unsigned b = lane; b < nk; b += 32) {  // one bin row per lane: byte-SIMD prefix
            uint4 *row = reinterpret_cast<uint4 *>(rows + b * 48);
            const uint4 q0 = row[0], q1 = row[1];
            unsigned w[8] = {q0.x, q0.y, q0.z, q0.w, q1.x, q1.y, q1.z, q1.w};
            unsigned base[8];
            unsigned run = 0;
  #pragma unroll
            for (int x = 0; x < 8; ++x) {
              const unsigned incl = w[x] * 0x01010101u;  // byte j = counts of lanes 4x .. 4x+j (<= 64)
              base[x] = run;
              run += incl >> 24;
              w[x] = incl - w[x];
            }
            row[0] = make_uint4(w[0], w[1], w[2], w[3]);
            row[1] = make_uint4(w[4], w[5], w[6], w[7]);
            row[2] = make_uint4(base[0] | (base[1] << 16), base[2] | (base[3] << 16), base[4] | (base[5] << 16),
                                base[6] | (base[7] << 16));
            myt[kb + b] = (unsigned short)run;
          }
          __syncwarp();
          const unsigned short *rows16 = reinterpret_cast<const unsigned short *>(rows);
  #pragma unroll
          for (int k = 0; k < kPerLane; ++k) {
            const unsigned key = kp[k] >> 16, rk = key - kb;
            if (key != kNoKey && (!MP || rk < nk)) kp[k] += rows[rk * 48 + lane] + rows16[rk * 24 + 16 + (lane >> 2)];
          }
          __syncwarp();  // the slot is free again
        };
        for (unsigned kb = 0; kb < nbins; kb += kLmMaxBins) rank_pass(kb, min(nbins - kb, kLmMaxBins));
      } else {  // one pass (the C2 path: kept as its own code, the lambda form spills 8 B here)
        uint4 *r4 = reinterpret_cast<uint4 *>(rows);
        for (unsigned q = lane; q < nbins * 3; q += 32) r4[q] = make_uint4(0, 0, 0, 0);
        __syncwarp();
#pragma unroll
        for (int k = 0; k < kPerLane; ++k) {
          const unsigned key = kp[k] >> 16;
          if (key != kNoKey) {
            unsigned char *ctr = rows + key * 48 + lane;
            const unsigned r = *ctr;
            *ctr = (unsigned char)(r + 1);
            kp[k] |= r;
          }
        }
        __syncwarp();
        for (unsigned b = lane; b < nbins; b += 32) {  // one bin row per lane: byte-SIMD prefix
          uint4 *row = reinterpret_cast<uint4 *>(rows + b * 48);
          const uint4 q0 = row[0], q1 = row[1];
          unsigned w[8] = {q0.x, q0.y, q0.z, q0.w, q1.x, q1.y, q1.z, q1.w};
          unsigned base[8];
          unsigned run = 0;
#pragma unroll
          for (int x = 0; x < 8; ++x) {
            const unsigned incl = w[x] * 0x01010101u;  // byte j = counts of lanes 4x .. 4x+j (<= 64)
            base[x] = run;
            run += incl >> 24;
            w[x] = incl - w[x];
          }
          row[0] = make_uint4(w[0], w[1], w[2], w[3]);
          row[1] = make_uint4(w[4], w[5], w[6], w[7]);
          row[2] = make_uint4(base[0] | (base[1] << 16), base[2] | (base[3] << 16), base[4] | (base[5] << 16),
                              base[6] | (base[7] << 16));
          myt[b] = (unsigned short)run;
        }
        __syncwarp();
        const unsigned short *rows16 = reinterpret_cast<const unsigned short *>(rows);
#pragma unroll
        for (int k = 0; k < kPerLane; ++k) {
          const unsigned key = kp[k] >> 16;
          if (key != kNoKey) kp[k] += rows[key * 48 + lane] + rows16[key * 24 + 16 + (lane >> 2)];
        }
        __syncwarp();  // the slot is free again
      }
    }
    PTM(3);
    // the next tile's records stream into the slot while this tile is published and written out
    cp_async_wait_all();
    __syncwarp();
    const bool early = warp >= kK1Warps / 2;  // slots outside the staged half
    if (early) {
      if (nxt != ~0u) prefetch_raw(dsm[par ^ 1]);
      cp_async_commit();
    }
    k1_publish(wsum[par], first, last, has, viol, kept);
    __syncthreads();  // B1 (the only CTA barrier per tile): summaries + bin totals of this tile
    PTM(4);
    {
      unsigned total = 0;
      if (is_win) {
        total = k1_bin_bases<KS>(p, tile, wt, myb);
        unsigned long long *sst = reinterpret_cast<unsigned long long *>(smem);
#pragma unroll
        for (int k = 0; k < kPerLane; ++k) {
          const unsigned key = kp[k] >> 16;
          if (key != kNoKey) sst[myb[key] + (kp[k] & 0xFFFFu)] = e[k];
        }
      }
      __syncthreads();  // B2: the tile's entries are in bin order in shared memory
      // the tile summary (serial, latency-bound) by the last warp, which is otherwise idle until
      // the next tile: wsum[par] is rewritten only after the next tile's barrier
      if (warp == kK1Warps - 1) k1_tile_summary(p, t, wsum[par]);
      if (!early) {
        if (is_win) {
          const uint4 *s4 = reinterpret_cast<const uint4 *>(smem);
          uint4 *d4 = reinterpret_cast<uint4 *>(p.stage + (size_t)tile * kTileS);
          for (unsigned q = threadIdx.x; q < (total + 1) / 2; q += kK1Threads / 2) d4[q] = s4[q];
        }
        asm volatile("bar.sync 1, %0;" ::"n"(kK1Threads / 2) : "memory");  // staged half read out
        if (nxt != ~0u) prefetch_raw(dsm[par ^ 1]);
        cp_async_commit();
      }
    }
    PTM(5);
    tile = nxt;
  }
  cp_async_wait_all();
  if (p.fuse_events) {  // then task-event tiles, claimed dynamically (K3 fused into K1): the event
    __shared__ unsigned s_et;  // work fills the partition's tail instead of competing with the fold
    const unsigned n_e = p.rte[p.W + 2];
    __syncthreads();  // every warp is done with the raw slots: they hold the event tile's counters
    for (;;) {
      if (threadIdx.x == 0) s_et = atomicAdd(p.unit_ctr + 2, 1u);
      __syncthreads();
      const unsigned et = s_et;
      if (et >= n_e) break;
      events_tile(p, et, smem);  // ends with a CTA barrier
    }
  }
}

// After B1, the whole CTA: bins in rows of blockDim.x (thread = bin, conflict-free); each bin's
// CTA base from one block scan per row, then every warp's base for the bin (earlier warps'
// counts added) written to wb[warp][bin] and the CTA base to the tile's soff row.  O(n_bins) per
// tile in total, instead of every warp scanning every bin (O(8 n_bins)): the cost that dominates
// the many-bin partition.  Ends with a CTA barrier; returns the tile's kept total.
__device__ __forceinline__ unsigned k1_bin_bases_cta(const Params &p, unsigned tile, const unsigned short *wt,
                                                     unsigned short *wb, unsigned *scratch) {
  const unsigned nbins = p.nbins;
  uint16_t *offs = p.soff + (size_t)tile * (nbins + 1);
  unsigned carry = 0;
  for (unsigned row = 0; row < nbins; row += blockDim.x) {
    const unsigned b = row + threadIdx.x;
    unsigned cnt[kK1Warps], T = 0;
#pragma unroll
    for (int w2 = 0; w2 < kK1Warps; ++w2) {
      cnt[w2] = b < nbins ? wt[(size_t)w2 * nbins + b] : 0u;
      T += cnt[w2];
    }
    unsigned tot;
    const unsigned base = carry + block_excl_scan(T, scratch, &tot);
    if (b < nbins) {
      offs[b] = (uint16_t)base;
      unsigned run = base;
#pragma unroll
      for (int w2 = 0; w2 < kK1Warps; ++w2) {
        wb[(size_t)w2 * nbins + b] = (unsigned short)run;
        run += cnt[w2];
      }
    }
    carry += tot;
  }
  if (threadIdx.x == 0) offs[nbins] = (uint16_t)carry;
  __syncthreads();
  return carry;
}

template <int BL>
__global__ void __launch_bounds__(kK1Threads) k_partition_mx(Params p) {
  extern __shared__ __align__(16) unsigned char smem[];
  __shared__ K1WarpSum wsum[kK1Warps];
  const unsigned tile = blockIdx.x;
  if (tile >= p.rts[p.W + 2]) return;  // grid sized by an upper bound (CTA-uniform)
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const unsigned lt = lanemask_lt();
  const unsigned nbins = p.nbins;
  unsigned long long *sbuf = reinterpret_cast<unsigned long long *>(smem);
  unsigned short *wt = reinterpret_cast<unsigned short *>(smem + (size_t)kTileS * 8);
  unsigned short *wb = reinterpret_cast<unsigned short *>(smem + (size_t)kTileS * 8 + k1_vec_bytes(nbins));
  unsigned short *myt = wt + (size_t)warp * nbins;
  unsigned short *myb = wb + (size_t)warp * nbins;
  const K1Tile t = k1_tile(p, tile);
  const bool is_win = t.g.window >= 0;
  const int sub0 = warp * kSub;
  const int4 *src = reinterpret_cast<const int4 *>(p.s) + t.start + sub0;
  if (is_win)
    for (unsigned q = lane; q < nbins; q += 32) myt[q] = 0;
  __syncwarp();
  unsigned long long e[kPerLane];
  unsigned kp[kPerLane];  // key << 16 | position within the warp's bin group
  unsigned long long first = 0, last = 0;
  bool has = false, viol = false;
  unsigned kept = 0;
#pragma unroll
  for (int h = 0; h < kPerLane; h += 4) {
    int4 v[4];
#pragma unroll
    for (int jj = 0; jj < 4; ++jj) {
      const int i = (h + jj) * 32 + lane;
      v[jj] = sub0 + i < t.n ? ld_stream(src + i) : make_int4(0, 0, 0, 0);
    }
#pragma unroll
    for (int jj = 0; jj < 4; ++jj) {
      const int j = h + jj;
      const int i = j * 32 + lane;
      const unsigned b = (unsigned)v[jj].z, lvl = (unsigned)v[jj].w & 0xFFFFu, c = (unsigned)v[jj].w >> 16;
      const unsigned capb = __ldg(p.cap + (b < p.nb ? b : 0u));
      const bool valid = (sub0 + i < t.n) & (b < p.nb) & (c == capb) & (lvl <= c);
      const unsigned long long off = (unsigned long long)(rec_ts(v[jj]) - t.lo);
      const unsigned vm = __ballot_sync(kFull, valid);
      const unsigned lower = vm & lt;
      const unsigned long long pv = __shfl_sync(kFull, off, lower ? 31 - __clz(lower) : lane);
      const unsigned long long nl = __shfl_sync(kFull, off, vm ? 31 - __clz(vm) : lane);
      const unsigned long long fo = __shfl_sync(kFull, off, vm ? __ffs(vm) - 1 : lane);
      viol |= valid & ((off >= t.wlen) | (lower ? off < pv : (has & (off < last))));
      if (vm) {
        if (!has) first = fo;
        has = true;
        last = nl;
      }
      const bool keep = valid & is_win;
      kept += keep;
      const unsigned key = keep ? (b >> BL) : kNoKey;
      unsigned pos = 0;
      if (is_win) {  // CTA-uniform
        // (per-bit ballots instead of MATCH measured equal on C3 / C4: the fallback is latency-bound)
        const unsigned peers = __match_any_sync(kFull, key);
        const unsigned basec = keep ? myt[key] : 0u;
        __syncwarp();
        if (keep && lane == __ffs(peers) - 1) myt[key] = (unsigned short)(basec + __popc(peers));
        __syncwarp();
        pos = basec + __popc(peers & lt);
      }
      kp[j] = (key << 16) | pos;
      e[j] = (off << (16 + BL)) | ((unsigned long long)lvl << BL) | (b & ((1u << BL) - 1u));
    }
  }
  k1_publish(wsum, first, last, has, viol, kept);
  __syncthreads();  // B1
  if (warp == 0) k1_tile_summary(p, t, wsum);
  if (!is_win) return;
  __shared__ unsigned bb_scratch[32];
  const unsigned total = k1_bin_bases_cta(p, tile, wt, wb, bb_scratch);
#pragma unroll
  for (int k = 0; k < kPerLane; ++k) {
    const unsigned key = kp[k] >> 16;
    if (key != kNoKey) sbuf[myb[key] + (kp[k] & 0xFFFFu)] = e[k];
  }
  __syncthreads();  // B2
  const uint4 *s4 = reinterpret_cast<const uint4 *>(sbuf);
  uint4 *d4 = reinterpret_cast<uint4 *>(p.stage + (size_t)tile * kTileS);
  for (unsigned q = threadIdx.x; q < (total + 1) / 2; q += kK1Threads) d4[q] = s4[q];
}

#endif  // RTM_TU_PARTITION

// ============================================================================================
// K1b (two-pass path: more than 170 bins, windows shorter than 2^32 ticks).  Pass 1 is the
// lane-major partition keyed by superbin (buffer_id >> 14, <= 64 keys), entries
// o << 32 | level << 16 | (buffer_id & 0x3FFF).  Here, one warp per (window, superbin) unit,
// claimed in window order: the unit's entries (its (tile, superbin) segments in ingest order)
// are re-partitioned by bin into (window, bin)-contiguous staging in the fold's entry format.
// Sweep 1 counts the unit's entries per bin (shared atomics) and fixes every bin's output range
// (woff); sweep 2 takes 512-entry chunks in ingest order, lane-major (lane l: chunk entries
// 16l .. 16l+15) as in K1, so the stable rank is a u8 (bin, lane) counter plus earlier lanes'
// counts (byte-SIMD prefix); the chunk is permuted by bin in shared memory and each bin's run is
// appended at its cursor.  The fold then reads one contiguous range per (window, bin) unit
// instead of one segment per tile of the window (C4: ~220 tiles per window, ~1 entry per
// segment).
// ============================================================================================
constexpr int kSubWarps = 8;
template <int BL>
struct SubSmem {
  static constexpr int kNB = 1 << (kSupLog - BL);  // bins per superbin: 64 (BL 8) or 128 (BL 7)
  unsigned long long buf[kSub];  // the loaded chunk (swizzled), then its permutation by bin
  unsigned char rows[kNB * 48];  // per bin: 32 u8 lane counters / in-word prefixes + 8 u16 word bases
  unsigned cur[kNB];             // sweep 1: counts; sweep 2: output cursor of each bin
  unsigned short cb[kNB];        // chunk base of each bin
  unsigned short ct[kNB];        // chunk count of each bin
  unsigned seg_base[32];
};

template <int BL, bool ENDK = false>  // ENDK: record the end keys of the range-parallel sequential fold
__global__ void __launch_bounds__(kSubWarps * 32, 2) k_subpart(Params p) {
  extern __shared__ __align__(16) unsigned char smem[];
  using SS = SubSmem<BL>;
  constexpr int kNB = SS::kNB, kPerB = kNB / 32;
  SS &Q = reinterpret_cast<SS *>(smem)[threadIdx.x >> 5];
  const int lane = threadIdx.x & 31;
  const unsigned lt = lanemask_lt(), le = (2u << lane) - 1u;
  const unsigned nsb = p.nsb, nbins = p.nbins, rs = nsb + 1;
  const unsigned n_units = p.W * nsb;
  // the unit's tile group [tg, tg + 32): flattened segment table -> Q.seg_base, returns the total
  auto group = [&](unsigned tg, unsigned t_hi, unsigned S, unsigned &my_end) -> unsigned {
    unsigned seg_lo = 0, seg_len = 0;
    if (tg + lane < t_hi) {
      const uint16_t *o = p.soff + (size_t)(tg + lane) * rs + S;
      seg_lo = __ldg(o);
      seg_len = (unsigned)__ldg(o + 1) - seg_lo;
    }
    unsigned pre = seg_len;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const unsigned y = __shfl_up_sync(kFull, pre, o);
      if (lane >= o) pre += y;
    }
    const unsigned nonempty = __ballot_sync(kFull, seg_len != 0);
    __syncwarp();  // the previous group's seg_base reads are done
    if (seg_len) Q.seg_base[__popc(nonempty & lt)] = (tg + lane) * (unsigned)kTileS + seg_lo - (pre - seg_len);
    my_end = seg_len ? pre : 0xFFFFFFFFu;
    __syncwarp();
    return __shfl_sync(kFull, pre, 31);
  };
  // staging index of flattened position c + lane of the group, ~0u past its end (c advances by
  // 32 per call).  Addresses first, loads after: a unit's loads are issued in batches, so the
  // warp waits for DRAM once per batch instead of once per 32 entries.
  auto addr = [&](unsigned c, unsigned total, unsigned my_end, unsigned &seg_before) -> unsigned {
    const unsigned x = my_end - c;
    const unsigned ends = __reduce_or_sync(kFull, x < 32u ? 1u << x : 0u);
    const unsigned sgi = seg_before + __popc(ends & le);
    seg_before += __popc(ends);
    const unsigned g = c + lane;
    return g < total ? Q.seg_base[sgi] + g : ~0u;
  };
  auto ld = [&](unsigned i) -> unsigned long long { return i != ~0u ? __ldcs(p.stage + i) : 0ull; };
  for (;;) {
    unsigned u = 0;
    if (lane == 0) u = atomicAdd(p.unit_ctr + 3, 1u);
    u = __shfl_sync(kFull, u, 0);
    if (u >= n_units) break;
    const unsigned w = u / nsb, S = u % nsb;
    // window range of the range-parallel sequential fold (seq_ranges == 1: none)
    const unsigned rng = ENDK && p.seq_ranges > 1u ? w / p.seq_range_len : ~0u;
    const unsigned t_lo = p.rts[w + 1], t_hi = p.rts[w + 2];
    // the unit's output base: the window's staging region + its entries of lower superbins
    unsigned before = 0;
    for (unsigned t = t_lo + lane; t < t_hi; t += 32) before += __ldg(p.soff + (size_t)t * rs + S);
    before = warp_sum(before);
    const unsigned ubase = t_lo * (unsigned)kTileS + before;
#pragma unroll
    for (int j = 0; j < kPerB; ++j) Q.cur[lane + 32 * j] = 0;
    __syncwarp();
    // ---- sweep 1: entries per bin
    for (unsigned tg = t_lo; tg < t_hi; tg += 32) {
      unsigned my_end;
      const unsigned total = group(tg, t_hi, S, my_end);
      unsigned sb = 0;
      for (unsigned c = 0; c < total; c += 256) {  // 8 steps per batch
        unsigned ix[8];
#pragma unroll
        for (int j = 0; j < 8; ++j) ix[j] = c + 32u * j < total ? addr(c + 32u * j, total, my_end, sb) : ~0u;
        unsigned long long v[8];
#pragma unroll
        for (int j = 0; j < 8; ++j) v[j] = ld(ix[j]);
#pragma unroll
        for (int j = 0; j < 8; ++j)
          if (ix[j] != ~0u) atomicAdd(&Q.cur[((unsigned)v[j] & ((1u << kSupLog) - 1u)) >> BL], 1u);
      }
    }
    __syncwarp();
    {  // bin ranges: exclusive scan of the counts (lane: kPerB consecutive bins)
      unsigned v[kPerB], tot = 0;
#pragma unroll
      for (int j = 0; j < kPerB; ++j) {
        v[j] = Q.cur[kPerB * lane + j];
        tot += v[j];
      }
      unsigned incl = tot;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const unsigned y = __shfl_up_sync(kFull, incl, o);
        if (lane >= o) incl += y;
      }
      unsigned run = ubase + incl - tot;
      unsigned *wo = p.woff + (size_t)w * (nbins + 1);
#pragma unroll
      for (int j = 0; j < kPerB; ++j) {
        const unsigned bin = S * kNB + kPerB * lane + j;
        if (bin < nbins) wo[bin] = run;
        Q.cur[kPerB * lane + j] = run;
        run += v[j];
      }
      if (S == nsb - 1 && lane == 31) wo[nbins] = run;  // the window's end
    }
    __syncwarp();
    // ---- sweep 2: stable scatter, 512-entry chunks
    for (unsigned tg = t_lo; tg < t_hi; tg += 32) {
      unsigned my_end;
      const unsigned total = group(tg, t_hi, S, my_end);
      unsigned sb = 0;
      for (unsigned c0 = 0; c0 < total; c0 += kSub) {
        const unsigned n = total - c0 < (unsigned)kSub ? total - c0 : (unsigned)kSub;
        // load (coalesced, lane-strided) into the swizzled chunk: entry i at row i >> 4, column
        // (i & 15) ^ (row & 15), so the lane-major read below is conflict-free per half-warp
        {
          unsigned ix[kPerLane];
          // warp-uniform condition: addr is a warp collective, called once per 32-position step
#pragma unroll
          for (int j = 0; j < kPerLane; ++j) ix[j] = 32u * j < n ? addr(c0 + 32u * j, total, my_end, sb) : ~0u;
          unsigned long long v[kPerLane];
#pragma unroll
          for (int j = 0; j < kPerLane; ++j) v[j] = ld(ix[j]);
#pragma unroll
          for (int j = 0; j < kPerLane; ++j) {
            const unsigned i = 32u * j + lane;
            Q.buf[(i & ~15u) | ((i & 15u) ^ ((i >> 4) & 15u))] = v[j];
          }
        }
        __syncwarp();
        uint4 *r4 = reinterpret_cast<uint4 *>(Q.rows);
        for (unsigned q = lane; q < (unsigned)kNB * 3; q += 32) r4[q] = make_uint4(0, 0, 0, 0);
        __syncwarp();
        unsigned long long e[kPerLane];
        unsigned kp[kPerLane];
#pragma unroll
        for (int k = 0; k < kPerLane; ++k) {
          e[k] = Q.buf[16 * lane + (k ^ (lane & 15))];
          const unsigned key = 16u * lane + k < n ? ((unsigned)e[k] & ((1u << kSupLog) - 1u)) >> BL : kNoKey;
          kp[k] = key << 16;
          if (key != kNoKey) {
            unsigned char *ctr = Q.rows + key * 48 + lane;
            const unsigned r = *ctr;
            *ctr = (unsigned char)(r + 1);
            kp[k] |= r;
          }
        }
        __syncwarp();
#pragma unroll
        for (int j = 0; j < kPerB; ++j) {  // one bin row per lane and step: byte-SIMD prefix
          const unsigned b = lane + 32 * j;
          uint4 *row = reinterpret_cast<uint4 *>(Q.rows + b * 48);
          const uint4 q0 = row[0], q1 = row[1];
          unsigned wv[8] = {q0.x, q0.y, q0.z, q0.w, q1.x, q1.y, q1.z, q1.w};
          unsigned base[8];
          unsigned run = 0;
#pragma unroll
          for (int x = 0; x < 8; ++x) {
            const unsigned incl = wv[x] * 0x01010101u;
            base[x] = run;
            run += incl >> 24;
            wv[x] = incl - wv[x];
          }
          row[0] = make_uint4(wv[0], wv[1], wv[2], wv[3]);
          row[1] = make_uint4(wv[4], wv[5], wv[6], wv[7]);
          row[2] = make_uint4(base[0] | (base[1] << 16), base[2] | (base[3] << 16), base[4] | (base[5] << 16),
                              base[6] | (base[7] << 16));
          Q.ct[b] = (unsigned short)run;
        }
        __syncwarp();
        {  // chunk bases: exclusive scan of the chunk counts
          unsigned v[kPerB], tot = 0;
#pragma unroll
          for (int j = 0; j < kPerB; ++j) {
            v[j] = Q.ct[kPerB * lane + j];
            tot += v[j];
          }
          unsigned incl = tot;
#pragma unroll
          for (int o = 1; o < 32; o <<= 1) {
            const unsigned y = __shfl_up_sync(kFull, incl, o);
            if (lane >= o) incl += y;
          }
          unsigned run = incl - tot;
#pragma unroll
          for (int j = 0; j < kPerB; ++j) {
            Q.cb[kPerB * lane + j] = (unsigned short)run;
            run += v[j];
          }
        }
        __syncwarp();
        const unsigned short *rows16 = reinterpret_cast<const unsigned short *>(Q.rows);
#pragma unroll
        for (int k = 0; k < kPerLane; ++k) {
          const unsigned key = kp[k] >> 16;
          if (key != kNoKey)
            Q.buf[Q.cb[key] + (kp[k] & 0xFFFFu) + Q.rows[key * 48 + lane] + rows16[key * 24 + 16 + (lane >> 2)]] = e[k];
        }
        __syncwarp();
        // copy out: each bin's run of the chunk appended at its cursor, in the fold's format
        for (unsigned q = lane; q < n; q += 32) {
          const unsigned long long x = Q.buf[q];
          const unsigned key = ((unsigned)x & ((1u << kSupLog) - 1u)) >> BL;
          const unsigned dst = Q.cur[key] + (q - Q.cb[key]);
          const unsigned long long lvl = (x >> 16) & 0xFFFFull;
          __stcg(p.stage2 + dst, ((x >> 32) << (16 + BL)) | (lvl << BL) | (x & ((1u << BL) - 1u)));
          if (ENDK && rng < p.seq_ranges - 1u)  // range-parallel sequential fold: latest level per buffer and range
            atomicMax(p.endkey + (size_t)rng * p.nb + (S << kSupLog) + ((unsigned)x & ((1u << kSupLog) - 1u)),
                      ((unsigned long long)(dst + 1u) << 16) | lvl);
        }
        __syncwarp();
#pragma unroll
        for (int j = 0; j < kPerB; ++j) Q.cur[lane + 32 * j] += Q.ct[lane + 32 * j];
        __syncwarp();
      }
    }
  }
}

// Persistence ranking key (rank mode MEAN): floor(I * 2^32 / c), exact.  Within a window the
// mean occupancy I / (c * W) orders like I / c; distinct ratios I1/c1 != I2/c2 differ by at least
// 1/(c1 c2) >= 2^-32 * 1.00003, so the floors differ: the key is exactly order-preserving.  Needs
// I / c < 2^32 (I <= c * W, windows shorter than 2^32 ticks).  m = floor(2^64 / c): q0 =
// floor(I m / 2^64) is floor(I / c) or one less (the error I eps / 2^64 < 1); one remainder test.
__device__ __forceinline__ unsigned long long mean_key(unsigned long long I, unsigned c,
                                                       const unsigned long long *rcp64) {
  if (c <= 1) return I << 32;
  const unsigned long long m = __ldg(rcp64 + c);
  unsigned long long q = __umul64hi(I, m), r = I - q * c;
  if (r >= c) ++q, r -= c;
  const unsigned long long x = r << 32;  // r < c <= 65535
  unsigned long long lo = __umul64hi(x, m);
  if (x - lo * c >= c) ++lo;
  return (q << 32) | lo;
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
// Per-buffer fold state, one 16-byte record so a chain head / tail moves it with ONE shared
// access: D (x, y), last | max << 16 (z), min | n16 << 16 (w).  last == 0xFFFF (never a valid
// level: capacity 65535 is reserved) marks a buffer untouched in the window; the sample count is
// hi[] * 65536 + n16 (hi[] low 16 bits, touched only when n16 wraps).  The offset of the first
// sample in the window is ts0 | (hi >> 16) << 32 (hi bits only for windows >= 2^32 ticks).  6.5 KB
// per warp: 8 CTAs of 4 warps per SM.
template <int BL>
struct FoldSmem {
  static constexpr int kB = 1 << BL;
  uint4 st[kB];
  unsigned ts0[kB];                // offset of the first kept sample in the window, low 32 bits
  unsigned hi[kB];                 // n_hi | ts0_hi << 16
  unsigned seg_base[32];           // staging index of each segment, minus its flattened start
  unsigned char owner[kB];         // duplicate detection: last lane that wrote each buffer slot
};
constexpr unsigned kUntouchedZ = 0xFFFFFFFFu;  // st.z of an untouched buffer
__device__ __forceinline__ bool st_touched(const uint4 &v) { return (v.z & 0xFFFFu) != 0xFFFFu; }
__device__ __forceinline__ unsigned long long st_D(const uint4 &v) {
  return ((unsigned long long)v.y << 32) | v.x;
}
// D and the first sample's offset (low 32 bits) of a touched state, either layout (ND: fold_chunk)
template <bool ND>
__device__ __forceinline__ unsigned long long st_Dn(const uint4 &v) { return ND ? (unsigned long long)v.x : st_D(v); }
template <bool ND, typename FS>
__device__ __forceinline__ unsigned st_ts0(const FS &S, const uint4 &v, unsigned l) { return ND ? v.y : S.ts0[l]; }

// One chunk of <= 32 consecutive records (ingest order) of one (window, bin) unit.  Records of
// the same buffer (peers, found with __match_any_sync) form a chain in lane order: each record's
// predecessor level is the previous peer's (shuffle) or, for the chain head, the buffer's state.
// Contributions are computed in parallel; the group's sum / max / min travel down the chain in
// `maxrank` shuffle steps and only the chain's last lane updates the shared state, so every
// state update in a chunk touches a distinct buffer.
// ND ("narrow D"): every registered capacity times every window length of the call
// is below 2^32.  D's partial sums then stay in [0, cap * Wlen] (Abel summation: D_j = l_j u_j +
// sum_{i<j} l_i (u_i - u_{i+1}) with u_i = t_end - ts_i non-increasing), so D is exact in unsigned
// 32-bit wrapping arithmetic, and st.y holds the first sample's offset instead of D's high word
// (one 16-byte state access per update, 32-bit products and chain shuffles).
template <bool NAR, int BL, bool ND = false>
__device__ __forceinline__ void fold_chunk(FoldSmem<BL> &S, int lane, unsigned lt, bool act, unsigned long long e,
                                           unsigned long long Wlen) {
  static_assert(!ND || NAR, "narrow D implies narrow windows");
  using DT = typename std::conditional<ND, unsigned, unsigned long long>::type;
  using OT = typename std::conditional<NAR, unsigned, unsigned long long>::type;
  const unsigned lid = (unsigned)(e & ((1u << BL) - 1u));
  const unsigned lvl = (unsigned)(e >> BL) & 0xFFFFu;
  const OT off = (OT)(e >> (16 + BL));
  // Peers = lanes holding the same buffer.  Most lanes hold a buffer no other lane of the chunk
  // holds, and __match_any_sync costs ~2 cycles of SM throughput per DISTINCT key in the warp
  // (tools/microbench.cu), so duplicates are found first through a shared-memory slot per
  // buffer (a lane whose write lost has a peer and tells the winner), and only duplicate lanes
  // present their real key to the match; the rest share one sentinel key.
  if (act) S.owner[lid] = (unsigned char)lane;
  __syncwarp();
  const unsigned win = act ? S.owner[lid] : (unsigned)lane;
  const bool lost = win != (unsigned)lane;
  const unsigned told = __reduce_or_sync(kFull, lost ? (1u << win) : 0u);
#ifndef RTM_FOLD_NODUP_FAST
#define RTM_FOLD_NODUP_FAST 1
#endif
  // (l - prev) * (t_end - ts): NAR one wide multiply; ND one 32-bit multiply (mod 2^32, exact at the end)
  auto contrib_of = [&](unsigned prev) -> DT {
    if constexpr (ND) return (unsigned)(lvl - prev) * (unsigned)((unsigned)Wlen - off);
    else if constexpr (NAR)
      return (unsigned long long)((long long)((int)lvl - (int)prev) * (long long)(unsigned)((unsigned)Wlen - off));
    else return (unsigned long long)((long long)((int)lvl - (int)prev) * (long long)(Wlen - off));
  };
  // the buffer state update of a chain tail (sum / mm / count over the chain, head's offset)
  // mm = max << 16 | (0xFFFF - min): one __vmaxu2 combines both halves
  auto update = [&](const uint4 &sv, bool c0, DT d, unsigned mm, unsigned n16, OT off0) {
    unsigned hi = mm >> 16, lo = (mm & 0xFFFFu) ^ 0xFFFFu;
    unsigned y;  // ND: first sample's offset; else D's high word
    if (c0) {
      hi = max(hi, sv.z >> 16);
      lo = min(lo, sv.w & 0xFFFFu);
      if constexpr (ND) {
        d += sv.x;
        y = sv.y;
      } else {
        d += st_D(sv);
      }
      n16 += sv.w >> 16;
      if (n16 > 0xFFFFu) {  // rare: more than 65535 samples of one buffer in one window
        S.hi[lid] += 1;
        n16 -= 0x10000u;
      }
    } else {
      if constexpr (ND) {
        y = (unsigned)off0;
      } else {
        S.ts0[lid] = (unsigned)off0;
        if constexpr (!NAR)
          if (off0 >> 32) S.hi[lid] += (unsigned)((unsigned long long)off0 >> 32) << 16;  // windows >= 2^32 ticks
      }
    }
    if constexpr (!ND) y = (unsigned)((unsigned long long)d >> 32);
    S.st[lid] = make_uint4((unsigned)d, y, lvl | (hi << 16), lo | (n16 << 16));
  };
  if (RTM_FOLD_NODUP_FAST && told == 0) {  // warp-uniform: every buffer of the chunk is distinct
    if (act) {  // each lane is its buffer's whole chain: no match, no chain propagation
      const uint4 sv = S.st[lid];
      const bool c0 = st_touched(sv);
      update(sv, c0, contrib_of(c0 ? (sv.z & 0xFFFFu) : 0u), (lvl << 16) | (lvl ^ 0xFFFFu), 1u, off);
    }
    __syncwarp();
    return;
  }
  const bool dup = lost | ((told >> lane) & 1u);
  const unsigned mk = __match_any_sync(kFull, dup ? lid : 0xFFFFFFFFu);
  const unsigned peers = dup ? mk : (1u << lane);
  const unsigned lower = peers & lt;
  const int pred = lower ? 31 - __clz(lower) : lane;
  const unsigned rank = __popc(lower);
  const bool tail = (peers >> lane) == 1u;
  const unsigned plv = __shfl_sync(kFull, lvl, pred);
  uint4 sv = make_uint4(0, 0, kUntouchedZ, 0);
  if (act && (!lower || tail)) sv = S.st[lid];  // chain heads need the level, tails the state
  const bool c0 = st_touched(sv);
  const unsigned prev = lower ? plv : (c0 ? (sv.z & 0xFFFFu) : 0u);
  const DT contrib = act ? contrib_of(prev) : (DT)0;
  DT sum = contrib;
  unsigned mm = (lvl << 16) | (lvl ^ 0xFFFFu);  // max << 16 | (0xFFFF - min) over the chain so far
  const unsigned maxrank = __reduce_max_sync(kFull, rank);
  // Pointer jumping along the chain: after s steps a lane holds the combination of its chain
  // elements at distance < 2^s, so ceil(log2(maxrank + 1)) steps (a hot buffer filling the chunk
  // - Zipf skew, C4 - takes 5 steps, not 31).  pj = predecessor lane | 0x100 while it has one.
  unsigned pj = (unsigned)pred | (lower ? 0x100u : 0u);
#pragma unroll 1
  for (unsigned d = 1; d <= maxrank; d <<= 1) {
    const int src = (int)(pj & 31u);
    const DT su = __shfl_sync(kFull, sum, src);
    const unsigned mu = __shfl_sync(kFull, mm, src);
    const unsigned pp = __shfl_sync(kFull, pj, src);
    if (pj & 0x100u) {
      sum += su;
      mm = __vmaxu2(mm, mu);
      pj = pp;
    }
  }
  const OT off0 = __shfl_sync(kFull, off, __ffs(peers) - 1);  // chain head's offset
  if (act && tail) update(sv, c0, sum, mm, rank + 1, off0);
  __syncwarp();
}

// Phase 2 of a fold unit (window w, bin), shared by both fold kernels: publish the window's last
// levels (kSent: untouched) and the phase-1 flag, resolve the carry-in L_in by decoupled
// look-back over earlier windows' published levels, finalize (integral, max / min with the
// carry-in, full bits, digest, mean-occupancy keys, watched buffers, the last window's table).
// S holds the unit's per-buffer phase-1 state: st (D, last | max << 16, min | n16 << 16), hi
// (n_hi | ts0_hi << 16) and ts0 (offset of the buffer's first kept sample in the window).
// digest term of one touched (window, buffer) (reading R17): odd-constant products
// of (I, n | id, levels | capacity), XOR, one fmix64 (splitmix64 finalizer)
__device__ __forceinline__ unsigned long long digest_term(unsigned long long I, unsigned cnt, unsigned bid, unsigned last,
                                                          unsigned mx, unsigned mn, unsigned capb) {
  unsigned long long h = (I * 0x9E3779B97F4A7C15ULL) ^ ((((unsigned long long)cnt << 32) | bid) * 0xC2B2AE3D27D4EB4FULL) ^
                         (((unsigned long long)last | ((unsigned long long)mx << 16) | ((unsigned long long)mn << 32) |
                           ((unsigned long long)capb << 48)) *
                          0x165667B19E3779F9ULL);
  h ^= h >> 30;
  h *= 0xbf58476d1ce4e5b9ULL;
  h ^= h >> 27;
  h *= 0x94d049bb133111ebULL;
  h ^= h >> 31;
  return h;
}

template <bool NAR, bool SPARSE, typename FS, bool CF = false, bool ND = false>
__device__ __forceinline__ void fold_finish(const Params &p, FS &S, unsigned w, unsigned bin,
                                            unsigned long long Wlen, int lane) {
  static_assert(!CF || (NAR && SPARSE), "compacted finalize: narrow windows, sparse units");
  {
    // ---- publish this window's last levels (kSent: untouched) and the phase-1 flag
    const unsigned b_base = bin * FS::kB;
    uint16_t *lw = p.lastlvl + (size_t)w * p.nb;
#pragma unroll
    for (int i = 0; i < FS::kB / 32; ++i) {
      const unsigned l = lane + 32 * i, b = b_base + l;
      if (b < p.nb) lw[b] = (uint16_t)(S.st[l].z & 0xFFFFu);  // 0xFFFF == kSent: untouched
    }
    // No per-lane fence: bar.warp.sync orders every lane's lastlvl stores before lane 0's
    // st.release.gpu, and release is cumulative (PTX memory model), so a reader that acquires the
    // flag sees them (measured: fold -2 %, the fence was 3.7 % of its stall samples).
    __syncwarp();
    if (lane == 0) st_release_u32(p.flags + (size_t)w * p.nbins + bin, p.epoch);
    // ---- phase 2: carry-in by look-back, finalize
    unsigned short lin[FS::kB / 32];
    unsigned need = 0;
#pragma unroll
    for (int i = 0; i < FS::kB / 32; ++i) {
      lin[i] = 0;
      if (b_base + lane + 32 * i < p.nb) need |= 1u << i;
    }
    int j = (int)w - 1;
    while (__any_sync(kFull, need != 0)) {
      if (j < 0) {
#pragma unroll
        for (int i = 0; i < FS::kB / 32; ++i)
          if (need & (1u << i)) lin[i] = __ldg(p.carry_in + b_base + lane + 32 * i);
        need = 0;
        break;
      }
#ifndef RTM_LB_STEP
#define RTM_LB_STEP 3  // measured (C3 fold / C5 fold per 20k windows): 2 -> 15.6 / 67.5 ms, 3 -> 14.7 / 60.5, 4 spills: 19.2 / 87.8
#endif
#ifndef RTM_LB_STEP_DENSE
#define RTM_LB_STEP_DENSE 1  // C2: 3 windows per step 704 us, 2 (spills) 727 us, 1 705 us - kept simple
#endif
      constexpr int kStep = SPARSE ? RTM_LB_STEP : RTM_LB_STEP_DENSE;  // windows per look-back step
      const int nwin = j + 1 < kStep ? j + 1 : kStep;   // windows j .. j - nwin + 1
      const int pair = nwin - 1;
      if (lane <= (unsigned)pair) {
        const unsigned *f = p.flags + (size_t)(j - lane) * p.nbins + bin;
        unsigned spins = 0;
#ifndef RTM_SPIN_RELAXED
#define RTM_SPIN_RELAXED 1
#endif
        // ld.acquire.gpu compiles to a strong load + CCTL.IVALL (the whole L1 invalidated) per
        // poll: spin relaxed, then ONE acquire of the flag (epochs are never overwritten within a
        // call, so it reads the published value and synchronizes with its release)
        while ((RTM_SPIN_RELAXED ? ld_relaxed_u32(f) : ld_acquire_u32(f)) != p.epoch) {
          __nanosleep(64);
          if (++spins > (1u << 25)) {  // ~seconds: never expected; fail loudly instead of hanging
            atomicOr(p.status, 4u);
            break;
          }
        }
        if (RTM_SPIN_RELAXED) (void)ld_acquire_u32(f);
#ifdef RTM_PHASE_TIMING
        if (p.dbg) atomicAdd(p.dbg + 6, (unsigned long long)spins);
#endif
      }
#ifdef RTM_PHASE_TIMING
      if (lane == 0 && p.dbg) atomicAdd(p.dbg + 0, 1ull);
#endif
      __syncwarp();
      const unsigned short *lj = p.lastlvl + (size_t)j * p.nb + b_base + lane;
      if constexpr (kStep > 1) {
        unsigned short v[kStep][FS::kB / 32];
#pragma unroll
        for (int d = 0; d < kStep; ++d)
#pragma unroll
          for (int i = 0; i < FS::kB / 32; ++i) {
            v[d][i] = kSent;
            if (d < nwin && (need & (1u << i))) v[d][i] = ld_relaxed_u16(lj - (size_t)d * p.nb + 32 * i);
          }
#pragma unroll
        for (int i = 0; i < FS::kB / 32; ++i) {
          if (need & (1u << i)) {
            unsigned short x = kSent;
#pragma unroll
            for (int d = kStep - 1; d >= 0; --d)
              if (v[d][i] != kSent) x = v[d][i];  // the most recent window holding a level wins
            if (x != kSent) {
              lin[i] = x;
              need &= ~(1u << i);
            }
          }
        }
        j -= nwin;
      } else {
#pragma unroll
        for (int i = 0; i < FS::kB / 32; ++i) {
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
    }
    unsigned long long dig = 0;
    unsigned touched = 0;
    // the window's statistics of buffer slot i (carry-in L_in = lin[i] resolved above)
    auto stat_of = [&](int i, unsigned long long &I, unsigned &mx, unsigned &mn, unsigned &last) -> unsigned {
      const unsigned l = lane + 32 * i, L = lin[i];
      const uint4 sv = S.st[l];
      const unsigned hw = S.hi[l];
      if (st_touched(sv)) {
        const unsigned hi = sv.z >> 16, lo = sv.w & 0xFFFFu;
        // NAR: the first sample's offset fits 32 bits (hw's upper half is reused below)
        I = (unsigned long long)L * (NAR ? (unsigned long long)st_ts0<ND>(S, sv, l)
                                         : (((unsigned long long)(hw >> 16) << 32) | S.ts0[l])) + st_Dn<ND>(sv);
        mx = hi > L ? hi : L;
        mn = lo < L ? lo : L;
        last = sv.z & 0xFFFFu;
        return ((hw & 0xFFFFu) << 16) + (sv.w >> 16);
      }
      I = (unsigned long long)L * Wlen;
      mx = mn = last = L;
      return 0u;
    };
    const unsigned nb = p.nb;
    const unsigned short *capp = p.cap;
    const bool nonempty_mode = p.hang_mode == RTM_HANG_NONEMPTY;
    if constexpr (CF) {  // compacted finalize (NAR, sparse units; launch_fold_bl decides)
      // Sparse units (C3, C4): many of the bin's buffers are untouched in the window.  Pass A
      // resolves every untouched cell (row, held-full bit from the carry-in, MEAN key) and
      // compacts the touched buffers into a list (the phase-1 owner slots are free now; each
      // touched buffer's carry-in goes to the upper half of its hi word, unused for narrow
      // windows); pass B finalizes the touched ones 32 at a time, so the digest runs on full
      // warps instead of once per slot for the few touched lanes.
      unsigned nt = 0;
#pragma unroll
      for (int i = 0; i < FS::kB / 32; ++i) {
        const unsigned l = lane + 32 * i, b = b_base + l;
        const bool t = b < nb && st_touched(S.st[l]);
        if (b < nb && !t) {
          const unsigned L = lin[i];
          lw[b] = (uint16_t)L;
          const unsigned capb = __ldg(capp + b);
          if (p.mkey) p.mkey[(size_t)w * nb + b] = mean_key((unsigned long long)L * Wlen, capb, p.rcp64);
          if (nonempty_mode ? L >= 1u : L == capb) {
            const unsigned c = __ldg(p.owner + b);
            atomicOr(p.anyfull + (size_t)w * p.ncw + (c >> 5), 1u << (c & 31));
          }
        }
        const unsigned m = __ballot_sync(kFull, t);
        if (t) {
          S.hi[l] |= (unsigned)lin[i] << 16;
          S.owner[nt + __popc(m & lanemask_lt())] = (unsigned char)l;
        }
        nt += __popc(m);
      }
      __syncwarp();
      for (unsigned q0 = 0; q0 < nt; q0 += 32) {
        const unsigned q = q0 + lane;
        if (q < nt) {
          const unsigned l = S.owner[q], b = b_base + l;
          const uint4 sv = S.st[l];
          const unsigned hw = S.hi[l], L = hw >> 16;
          const unsigned hi = sv.z >> 16, lo = sv.w & 0xFFFFu;
          const unsigned long long I = (unsigned long long)L * st_ts0<ND>(S, sv, l) + st_Dn<ND>(sv);
          const unsigned mx = hi > L ? hi : L, mn = lo < L ? lo : L, last = sv.z & 0xFFFFu;
          const unsigned cnt = ((hw & 0xFFFFu) << 16) + (sv.w >> 16);
          const unsigned capb = __ldg(capp + b);
          if (p.mkey) p.mkey[(size_t)w * nb + b] = mean_key(I, capb, p.rcp64);
          if (nonempty_mode ? mn >= 1u : mn == capb) {
            const unsigned c = __ldg(p.owner + b);
            atomicOr(p.anyfull + (size_t)w * p.ncw + (c >> 5), 1u << (c & 31));
          }
          const unsigned bid = p.gid ? __ldg(p.gid + b) : b;
          dig += digest_term(I, cnt, bid, last, mx, mn, capb);
        }
      }
      touched = lane == 0 ? nt : 0u;  // summed over the warp below
      __syncwarp();
      // the last-window / value-monitor pass below reads the carry-in from lin[] and the
      // first-sample offset from ts0 only (NAR), so the reused hi bits do not matter
    } else {
#pragma unroll
    for (int i = 0; i < FS::kB / 32; ++i) {
      const unsigned b = b_base + lane + 32 * i;
      if (b >= nb) continue;
      unsigned long long I;
      unsigned mx, mn, last;
      const unsigned cnt = stat_of(i, I, mx, mn, last);
      if (!cnt) lw[b] = (uint16_t)last;  // resolve the untouched cell
      const unsigned capb = __ldg(capp + b);
      if (p.mkey) p.mkey[(size_t)w * nb + b] = mean_key(I, capb, p.rcp64);
      if (p.hang_mode == RTM_HANG_NONEMPTY ? mn >= 1u : mn == capb) {  // held the whole window
        const unsigned c = __ldg(p.owner + b);
        atomicOr(p.anyfull + (size_t)w * p.ncw + (c >> 5), 1u << (c & 31));
      }
      if (cnt) {
        // digest term: odd-constant products of (I, n|b, levels), XOR, one fmix64
        const unsigned bid = p.gid ? __ldg(p.gid + b) : b;  // the digest names buffers by global id
        unsigned long long h = (I * 0x9E3779B97F4A7C15ULL) ^
                               ((((unsigned long long)cnt << 32) | bid) * 0xC2B2AE3D27D4EB4FULL) ^
                               (((unsigned long long)last | ((unsigned long long)mx << 16) |
                                 ((unsigned long long)mn << 32) | ((unsigned long long)capb << 48)) *
                                0x165667B19E3779F9ULL);
        h ^= h >> 30;
        h *= 0xbf58476d1ce4e5b9ULL;
        h ^= h >> 27;
        h *= 0x94d049bb133111ebULL;
        h ^= h >> 31;
        dig += h;
        ++touched;
      }
    }
    }
    // rare, uniform: the call's last window (per-buffer table, next call's carry) and the value
    // monitor's watched buffers - a second pass, so the loop above stays small
    const bool last_window = (w == p.W - 1);
    if (last_window || p.n_watch) {
#pragma unroll
      for (int i = 0; i < FS::kB / 32; ++i) {
        const unsigned b = b_base + lane + 32 * i;
        if (b >= nb) continue;
        int wq = -1;  // value monitor slot of b (at most RTM_WATCH_MAX compares)
        for (unsigned q = 0; q < p.n_watch; ++q)
          if (p.watch[q] == b) wq = (int)q;
        if (!last_window && wq < 0) continue;
        unsigned long long I;
        unsigned mx, mn, last;
        const unsigned cnt = stat_of(i, I, mx, mn, last);
        const unsigned capb = __ldg(capp + b);
        rtm_buffer_stat st;
        st.integral = (int64_t)I;
        st.last = (uint16_t)last;
        st.max = (uint16_t)mx;
        st.min = (uint16_t)mn;
        st.capacity = (uint16_t)capb;
        st.n_samples = cnt;
        st.reserved = __ldg(p.elig + b);
        st.mean_occ = Wlen ? __ddiv_rn((double)(long long)I, (double)((long long)capb * (long long)Wlen)) : 0.0;
        if (wq >= 0) p.wstat[(size_t)w * RTM_WATCH_MAX + wq] = st;
        if (last_window) {
          p.bstat[b] = st;
          p.carry_out[b] = (uint16_t)last;
        }
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

// Phase 1 of a fold unit (window w, bin): the (tile, bin) segments of window w flattened into one
// stream of 32-sample chunks, each folded by fold_chunk into S (carry-in left symbolic).
template <bool NAR, int BL, bool ND = false>
__device__ __forceinline__ void fold_phase1(const Params &p, FoldSmem<BL> &S, unsigned w, unsigned bin,
                                            unsigned long long Wlen, int lane, unsigned lt) {
  if (p.woff) {  // two-pass path: the unit's entries are one contiguous range
    const unsigned *wo = p.woff + (size_t)w * (p.nbins + 1) + bin;
    const unsigned lo = __ldg(wo), total = __ldg(wo + 1) - lo;
    const unsigned long long *src = p.stage2 + lo;
    auto fetch = [&](unsigned c) -> unsigned long long { return c + lane < total ? __ldcs(src + c + lane) : 0ull; };
    unsigned long long e0 = fetch(0), e1 = fetch(32);
    for (unsigned c = 0; c < total; c += 32) {
      const unsigned long long en = fetch(c + 64);
      fold_chunk<NAR, BL, ND>(S, lane, lt, c + lane < total, e0, Wlen);
      e0 = e1;
      e1 = en;
    }
    return;
  }
  const unsigned t_lo = p.rts[w + 1], t_hi = p.rts[w + 2];
  {
    // ---- phase 1: the (tile, bin) segments of window w, flattened into one stream of chunks
    for (unsigned tg = t_lo; tg < t_hi; tg += 32) {
      unsigned seg_lo = 0, seg_len = 0;
      if (tg + lane < t_hi) {
        const uint16_t *o = p.soff + (size_t)(tg + lane) * (p.nbins + 1) + bin;
        seg_lo = __ldg(o);
        seg_len = (unsigned)__ldg(o + 1) - seg_lo;
      }
      unsigned pre = seg_len;  // inclusive prefix of segment lengths over lanes
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const unsigned y = __shfl_up_sync(kFull, pre, o);
        if (lane >= o) pre += y;
      }
      const unsigned total = __shfl_sync(kFull, pre, 31);
      // per-warp table of the NON-EMPTY segments (compacted, so their ends are strictly
      // increasing): staging index of each segment minus its flattened start.  The segment of
      // flattened position g is the number of segment ends <= g: per 32-position chunk, one
      // OR-reduction marks the ends inside the chunk and each lane counts the marks at or below it.
      const unsigned nonempty = __ballot_sync(kFull, seg_len != 0);
      if (seg_len) S.seg_base[__popc(nonempty & lt)] = (tg + lane) * (unsigned)kTileS + seg_lo - (pre - seg_len);
      const unsigned my_end = seg_len ? pre : 0xFFFFFFFFu;
      const unsigned le = (2u << lane) - 1u;  // lanes <= this one
      __syncwarp();
      unsigned seg_before = 0;  // segments ending at or before the current chunk's first position
      auto fetch = [&](unsigned c) -> unsigned long long {
        const unsigned x = my_end - c;
        const unsigned ends = __reduce_or_sync(kFull, x < 32u ? 1u << x : 0u);
        const unsigned sgi = seg_before + __popc(ends & le);
        seg_before += __popc(ends);
        const unsigned g = c + lane;
        if (g >= total) return 0ull;
        return __ldcg(p.stage + (S.seg_base[sgi] + g));
      };
      // 2-deep software pipeline over the staging reads (measured on C2: depth 2 709 us, 3 715 us,
      // 4 719 us, 6 727 us - deeper costs registers the chunk logic needs; depth 1: 863 us)
      unsigned long long e0 = fetch(0), e1 = fetch(32);
      for (unsigned c = 0; c < total; c += 32) {
        const unsigned long long en = fetch(c + 64);
        fold_chunk<NAR, BL, ND>(S, lane, lt, c + lane < total, e0, Wlen);
        e0 = e1;
        e1 = en;
      }
    }
  }
}

// SPARSE (few samples per unit: C3-C5 shapes): many of a unit's 256 buffers are untouched in
// several consecutive windows, so the look-back walks several windows; it takes RTM_LB_STEP of
// them per step (their flags waited for by as many lanes, all rows loaded before any is used),
// dividing the dependent round trips.  A separate instantiation: the dense (C2) code is unchanged.
template <bool NAR, bool SPARSE, int BL, bool CF = false, bool ND = false>
__global__ void __launch_bounds__(kFoldWarps * 32, 32 / kFoldWarps) k_fold(Params p) {
  extern __shared__ __align__(16) unsigned char smem[];
  using FS = FoldSmem<BL>;
  FS &S = reinterpret_cast<FS *>(smem)[threadIdx.x >> 5];
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
#pragma unroll
    for (int i = 0; i < FS::kB / 32; ++i) {
      S.st[lane + 32 * i] = make_uint4(0, 0, kUntouchedZ, 0);
      S.hi[lane + 32 * i] = 0;
    }
    __syncwarp();
    fold_phase1<NAR, BL, ND>(p, S, w, bin, Wlen, lane, lt);
    fold_finish<NAR, SPARSE, FoldSmem<BL>, CF, ND>(p, S, w, bin, Wlen, lane);
  }
}

// ============================================================================================
// K2 for very sparse calls (C5: ~0.02 kept samples per buffer and window): one warp per bin
// walks ALL windows of the call in order, so every buffer's carry-in is known when its window is
// finalized (no published rows to look back through) and the per-window work is proportional to
// the window's records, not to the bin's 256 buffers:
//   - the window's samples are folded by fold_phase1 (as in k_fold);
//   - only touched buffers are finalized (integral, max / min with the carry-in, digest, count),
//     their carried level advanced and their state reset;
//   - every buffer still gets its cell of the window's last-level row (the top-k ranks all
//     buffers) and its held-full bit (hang, R9), from the carried level when untouched.
// Lane l owns buffers l + 32 i (i < 8) of the bin; their capacities and owners stay in registers
// for the whole call, their carried levels in shared memory.  Rank mode MEAN (a 64-bit key per
// buffer and window) keeps the windowed k_fold.
// ============================================================================================
template <int BL>
struct FoldSeqSmem {
  static constexpr int kB = 1 << BL, kPer = kB / 32, kQ = 64;
  FoldSmem<BL> f;
  // touched (window, buffer) results awaiting their finalize, 32 at a time: state; hi word, window,
  // lid | carried level << 16, first sample's offset (wide layout)
  uint4 qst[kQ];
  uint4 qmeta[kQ];
  unsigned short lvl[kB];   // carried level of every buffer of the bin
  unsigned short list[kB];  // the window's touched buffers (compacted)
  unsigned short capS[kB];  // capacities and owners of the bin (the touched finalize reads them)
  unsigned ownS[kB];
  unsigned tmask[kPer];     // the window's touched buffers (bit lid)
};

template <bool NAR, int BL, bool ND = false>
__global__ void __launch_bounds__(kFoldWarps * 32) k_fold_seq(Params p) {
  extern __shared__ __align__(16) unsigned char smem[];
  using QS = FoldSeqSmem<BL>;
  constexpr int kB = QS::kB, kPer = QS::kPer;
  QS &Q = reinterpret_cast<QS *>(smem)[threadIdx.x >> 5];
  FoldSmem<BL> &S = Q.f;
  const int lane = threadIdx.x & 31;
  const unsigned lt = lanemask_lt();
  const bool nonempty_mode = p.hang_mode == RTM_HANG_NONEMPTY;
  const unsigned n_ranges = p.seq_ranges > 1u ? p.seq_ranges : 1u;
  for (;;) {
    unsigned u = 0;
    if (lane == 0) u = atomicAdd(p.unit_ctr, 1u);
    u = __shfl_sync(kFull, u, 0);
    if (u >= p.nbins * n_ranges) break;
    // unit = (bin, range of windows): range r starts from the carried levels at the end of range
    // r - 1, i.e. each buffer's latest kept sample in the ranges before it (k_subpart's end keys),
    // else the call's carry-in
    const unsigned bin = u % p.nbins, rg = u / p.nbins;
    const unsigned w_lo = n_ranges > 1u ? rg * p.seq_range_len : 0u;
    const unsigned w_hi = n_ranges > 1u ? min(p.W, w_lo + p.seq_range_len) : p.W;
    const unsigned b_base = bin * (unsigned)kB;
    // this lane's contiguous buffers kPer lane .. kPer lane + kPer - 1 (row stores, held-full bits)
    const unsigned c0 = b_base + kPer * lane;
    const bool vec = (p.nb & (kPer - 1)) == 0;  // aligned row segments
    unsigned capv[kPer], ownv[kPer];
#pragma unroll
    for (int j = 0; j < kPer; ++j) {
      const unsigned b = c0 + j;
      capv[j] = b < p.nb ? __ldg(p.cap + b) : 0xFFFFu;
      ownv[j] = b < p.nb ? __ldg(p.owner + b) : 0;
    }
#pragma unroll
    for (int i = 0; i < kPer; ++i) {
      const unsigned l = lane + 32 * i, b = b_base + l;
      S.st[l] = make_uint4(0, 0, kUntouchedZ, 0);
      S.hi[l] = 0;
      unsigned short L = b < p.nb ? __ldg(p.carry_in + b) : 0;
      for (int r2 = (int)rg - 1; r2 >= 0 && b < p.nb; --r2) {
        const unsigned long long k = __ldcg(p.endkey + (size_t)r2 * p.nb + b);
        if (k) {
          L = (unsigned short)(k & 0xFFFFu);
          break;
        }
      }
      Q.lvl[l] = L;
      Q.capS[l] = b < p.nb ? __ldg(p.cap + b) : 0xFFFFu;
      Q.ownS[l] = b < p.nb ? __ldg(p.owner + b) : 0;
    }
    __syncwarp();
    // finalize queue entries [base, base + m), one per lane: integral, max / min with the carried
    // level, digest (added to its window's sum), held-full bit, the call's table / value monitor
    unsigned qn = 0;
    auto flush = [&](unsigned base, unsigned m) {
      if ((unsigned)lane < m) {
        const uint4 sv = Q.qst[base + lane], mt = Q.qmeta[base + lane];
        const unsigned hw = mt.x, w = mt.y, l = mt.z & 0xFFFFu, L = mt.z >> 16, b = b_base + l;
        const unsigned cnt = ((hw & 0xFFFFu) << 16) + (sv.w >> 16);
        const unsigned hi = sv.z >> 16, lo = sv.w & 0xFFFFu;
        const unsigned long long I =
            (unsigned long long)L * (ND ? (unsigned long long)sv.y : (((unsigned long long)(hw >> 16) << 32) | mt.w)) +
            st_Dn<ND>(sv);
        const unsigned mx = hi > L ? hi : L, mn = lo < L ? lo : L, last = sv.z & 0xFFFFu;
        const unsigned capb = Q.capS[l];
        const unsigned bid = p.gid ? __ldg(p.gid + b) : b;
        atomicAdd(p.win + WF_DIGEST * p.W + w, digest_term(I, cnt, bid, last, mx, mn, capb));
        if (nonempty_mode ? mn >= 1u : mn == capb) {  // held the whole window
          const unsigned c = Q.ownS[l];
          atomicOr(p.anyfull + (size_t)w * p.ncw + (c >> 5), 1u << (c & 31));
        }
        const bool last_window = (w == p.W - 1);
        if (last_window || p.n_watch) {  // rare: the call's table, the value monitor
          int wq = -1;
          for (unsigned k2 = 0; k2 < p.n_watch; ++k2)
            if (p.watch[k2] == b) wq = (int)k2;
          if (last_window || wq >= 0) {
            const unsigned long long Wlen = (unsigned long long)(p.T[w + 1] - p.T[w]);
            rtm_buffer_stat st;
            st.integral = (int64_t)I;
            st.last = (uint16_t)last;
            st.max = (uint16_t)mx;
            st.min = (uint16_t)mn;
            st.capacity = (uint16_t)capb;
            st.n_samples = cnt;
            st.reserved = __ldg(p.elig + b);
            st.mean_occ = Wlen ? __ddiv_rn((double)(long long)I, (double)((long long)capb * (long long)Wlen)) : 0.0;
            if (wq >= 0) p.wstat[(size_t)w * RTM_WATCH_MAX + wq] = st;
            if (last_window) {
              p.bstat[b] = st;
              p.carry_out[b] = (uint16_t)last;
            }
          }
        }
      }
      __syncwarp();
    };
    // finalize of window w (its samples are folded into S): touched buffers queued, the
    // last-level row, held-full bits of the untouched ones, the window's touched count
    auto finalize = [&](unsigned w, unsigned long long Wlen) {
      const bool last_window = (w == p.W - 1);
        // ---- compact the touched buffers (owner-strided scan of the state)
        unsigned nt = 0;
#pragma unroll
        for (int i = 0; i < kPer; ++i) {
          const bool t = st_touched(S.st[lane + 32 * i]);
          const unsigned m = __ballot_sync(kFull, t);
          if (t) Q.list[nt + __popc(m & lt)] = (unsigned short)(lane + 32 * i);
          if (lane == 0) Q.tmask[i] = m;
          nt += __popc(m);
        }
        __syncwarp();
        // ---- queue the touched buffers (state, carried level, window), advance their carried
        // level and reset their state; the queue is finalized 32 entries at a time (flush), so
        // the digest runs on full warps across windows instead of a few lanes per window
        for (unsigned q0 = 0; q0 < nt; q0 += 32) {
          const unsigned n = nt - q0 < 32u ? nt - q0 : 32u;
          if (qn + n > (unsigned)QS::kQ) {  // warp-uniform: make room
            flush(0, qn);
            qn = 0;
          }
          if ((unsigned)lane < n) {
            const unsigned l = Q.list[q0 + lane];
            const uint4 sv = S.st[l];
            Q.qst[qn + lane] = sv;
            Q.qmeta[qn + lane] = make_uint4(S.hi[l], w, l | ((unsigned)Q.lvl[l] << 16), ND ? 0u : S.ts0[l]);
            Q.lvl[l] = (unsigned short)(sv.z & 0xFFFFu);
            S.st[l] = make_uint4(0, 0, kUntouchedZ, 0);
            S.hi[l] = 0;
          }
          qn += n;
          __syncwarp();
          if (qn >= 32u) {
            flush(qn - 32u, 32u);
            qn -= 32u;
          }
        }
        __syncwarp();
        // ---- the window's last-level row (every buffer) and the untouched buffers' held-full bits
        uint16_t *lw = p.lastlvl + (size_t)w * p.nb;
        unsigned lvw[kPer / 2];  // levels of c0 .. c0 + kPer - 1, two per word
        if constexpr (kPer == 8) {
          const uint4 v = reinterpret_cast<const uint4 *>(Q.lvl)[lane];
          lvw[0] = v.x; lvw[1] = v.y; lvw[2] = v.z; lvw[3] = v.w;
          if (vec && c0 < p.nb) reinterpret_cast<uint4 *>(lw + b_base)[lane] = v;
        } else {
          const uint2 v = reinterpret_cast<const uint2 *>(Q.lvl)[lane];
          lvw[0] = v.x; lvw[1] = v.y;
          if (vec && c0 < p.nb) reinterpret_cast<uint2 *>(lw + b_base)[lane] = v;
        }
        if (!vec) {
#pragma unroll
          for (int j = 0; j < kPer; ++j)
            if (c0 + j < p.nb) lw[c0 + j] = (uint16_t)(lvw[j >> 1] >> (16 * (j & 1)));
        }
        const unsigned tb8 = (Q.tmask[(kPer * lane) >> 5] >> ((kPer * lane) & 31)) & ((1u << kPer) - 1u);
        // untouched buffers held full (non-empty) by their carried level; the touched ones were
        // decided above from their window minimum
#pragma unroll
        for (int j = 0; j < kPer; ++j) {
          const unsigned L = (lvw[j >> 1] >> (16 * (j & 1))) & 0xFFFFu;
          if (!((tb8 >> j) & 1u) && c0 + j < p.nb && (nonempty_mode ? L >= 1u : L == capv[j]))
            atomicOr(p.anyfull + (size_t)w * p.ncw + (ownv[j] >> 5), 1u << (ownv[j] & 31));
        }
        if (last_window || p.n_watch) {  // rare: untouched buffers' statistics
#pragma unroll
          for (int j = 0; j < kPer; ++j) {
            const unsigned b = c0 + j;
            if (b >= p.nb || ((tb8 >> j) & 1u)) continue;
            int wq = -1;
            for (unsigned k2 = 0; k2 < p.n_watch; ++k2)
              if (p.watch[k2] == b) wq = (int)k2;
            if (!last_window && wq < 0) continue;
            const unsigned L = Q.lvl[kPer * lane + j];
            rtm_buffer_stat st;
            st.integral = (int64_t)((unsigned long long)L * Wlen);
            st.last = st.max = st.min = (uint16_t)L;
            st.capacity = (uint16_t)capv[j];
            st.n_samples = 0;
            st.reserved = __ldg(p.elig + b);
            st.mean_occ = Wlen ? __ddiv_rn((double)(long long)((unsigned long long)L * Wlen),
                                           (double)((long long)capv[j] * (long long)Wlen)) : 0.0;
            if (wq >= 0) p.wstat[(size_t)w * RTM_WATCH_MAX + wq] = st;
            if (last_window) {
              p.bstat[b] = st;
              p.carry_out[b] = (uint16_t)L;
            }
          }
        }
        if (lane == 0 && nt) atomicAdd(p.win + WF_TOUCHED * p.W + w, (unsigned long long)nt);
        __syncwarp();
    };
    // Software pipeline over the windows: while window w's staging entries and window w+1's
    // segment offsets are in flight, window w-1 is finalized (a window's chain of dependent
    // loads - tile range, segment offsets, entries - would otherwise stall the warp every window).
    // Fast path: a window's segments for this bin span <= 32 tiles; else fold_phase1.
    if (p.woff) {  // two-pass path: one contiguous range per (window, bin)
      const unsigned rs = p.nbins + 1;
      unsigned n_lo = __ldg(p.woff + (size_t)w_lo * rs + bin), n_hi = __ldg(p.woff + (size_t)w_lo * rs + bin + 1);
      bool pend = false;
      unsigned pw = 0;
      unsigned long long pWlen = 0;
      for (unsigned w = w_lo; w < w_hi; ++w) {
        const long long tb = p.T[w], te = p.T[w + 1];
        const unsigned long long Wlen = (unsigned long long)(te - tb);
        const unsigned total = n_hi - n_lo;
        const unsigned long long *src = p.stage2 + n_lo;
        auto fetch = [&](unsigned c) -> unsigned long long { return c + lane < total ? __ldcs(src + c + lane) : 0ull; };
        unsigned long long e0 = fetch(0), e1 = total > 32u ? fetch(32) : 0ull;
        if (w + 1 < w_hi) {  // the next window's range (in flight during the finalize)
          n_lo = __ldg(p.woff + (size_t)(w + 1) * rs + bin);
          n_hi = __ldg(p.woff + (size_t)(w + 1) * rs + bin + 1);
        }
        if (pend) finalize(pw, pWlen);
        for (unsigned c = 0; c < total; c += 32) {
          const unsigned long long en = c + 64 < total ? fetch(c + 64) : 0ull;
          fold_chunk<NAR, BL, ND>(S, lane, lt, c + lane < total, e0, Wlen);
          e0 = e1;
          e1 = en;
        }
        __syncwarp();
        pend = true;
        pw = w;
        pWlen = Wlen;
      }
      if (pend) finalize(pw, pWlen);
      flush(0, qn);
      continue;
    }
    unsigned n_tlo = p.rts[1], n_thi = p.rts[2];
    unsigned n_lo = 0, n_len = 0;
    bool n_ok = n_thi - n_tlo <= 32u;
    if (n_ok && n_tlo + lane < n_thi) {
      const uint16_t *o = p.soff + (size_t)(n_tlo + lane) * (p.nbins + 1) + bin;
      n_lo = __ldg(o);
      n_len = (unsigned)__ldg(o + 1) - n_lo;
    }
    bool pend = false;
    unsigned pw = 0;
    unsigned long long pWlen = 0;
    for (unsigned w = 0; w < p.W; ++w) {
      const long long tb = p.T[w], te = p.T[w + 1];
      const unsigned long long Wlen = (unsigned long long)(te - tb);
      if (n_ok) {
        const unsigned t_lo = n_tlo, seg_lo = n_lo, seg_len = n_len;
        // flatten window w's segments (one group of <= 32 tiles)
        unsigned pre = seg_len;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
          const unsigned y = __shfl_up_sync(kFull, pre, o);
          if (lane >= o) pre += y;
        }
        const unsigned total = __shfl_sync(kFull, pre, 31);
        const unsigned nonempty = __ballot_sync(kFull, seg_len != 0);
        if (seg_len) S.seg_base[__popc(nonempty & lt)] = (t_lo + lane) * (unsigned)kTileS + seg_lo - (pre - seg_len);
        const unsigned my_end = seg_len ? pre : 0xFFFFFFFFu;
        const unsigned le = (2u << lane) - 1u;
        __syncwarp();
        unsigned seg_before = 0;
        auto fetch = [&](unsigned c) -> unsigned long long {
          const unsigned x = my_end - c;
          const unsigned ends = __reduce_or_sync(kFull, x < 32u ? 1u << x : 0u);
          const unsigned sgi = seg_before + __popc(ends & le);
          seg_before += __popc(ends);
          const unsigned g = c + lane;
          if (g >= total) return 0ull;
          return __ldcg(p.stage + (S.seg_base[sgi] + g));
        };
        unsigned long long e0 = fetch(0), e1 = total > 32u ? fetch(32) : 0ull;  // usually one chunk
        // next window's tile range and this lane's segment (in flight during the finalize)
        if (w + 1 < p.W) {
          n_tlo = n_thi;
          n_thi = p.rts[w + 3];
          n_ok = n_thi - n_tlo <= 32u;
          n_lo = n_len = 0;
          if (n_ok && n_tlo + lane < n_thi) {
            const uint16_t *o = p.soff + (size_t)(n_tlo + lane) * (p.nbins + 1) + bin;
            n_lo = __ldg(o);
            n_len = (unsigned)__ldg(o + 1) - n_lo;
          }
        }
        if (pend) finalize(pw, pWlen);
        for (unsigned c = 0; c < total; c += 32) {
          const unsigned long long en = c + 64 < total ? fetch(c + 64) : 0ull;
          fold_chunk<NAR, BL, ND>(S, lane, lt, c + lane < total, e0, Wlen);
          e0 = e1;
          e1 = en;
        }
        __syncwarp();
      } else {  // many tiles in one window: the general phase 1, no overlap
        if (pend) finalize(pw, pWlen);
        fold_phase1<NAR, BL, ND>(p, S, w, bin, Wlen, lane, lt);
        __syncwarp();
        if (w + 1 < p.W) {
          n_tlo = p.rts[w + 2];
          n_thi = p.rts[w + 3];
          n_ok = n_thi - n_tlo <= 32u;
          n_lo = n_len = 0;
          if (n_ok && n_tlo + lane < n_thi) {
            const uint16_t *o = p.soff + (size_t)(n_tlo + lane) * (p.nbins + 1) + bin;
            n_lo = __ldg(o);
            n_len = (unsigned)__ldg(o + 1) - n_lo;
          }
        }
      }
      pend = true;
      pw = w;
      pWlen = Wlen;
    }
    if (pend) finalize(pw, pWlen);
    flush(0, qn);
  }
}

#ifndef RTM_TU_PARTITION  // (to the end of the file but the partition launchers)
// ============================================================================================
// K4: cross-tile order check.  Every tile has its in-tile verdict (flag bit 1: range / order
// inside the tile) and the offsets of its first / last field-valid record.  The field-valid
// stream is non-decreasing iff every tile passes its own check and starts at or after the last
// field-valid record of the nearest earlier tile that has one, so each tile is checked
// independently (one thread per tile; the back-scan over tiles without valid records is
// normally zero steps).  Sample tiles first, then event tiles, in one launch.
// ============================================================================================
__global__ void k_order_check(Params p) {
  const unsigned ns = p.rts[p.W + 2] < p.n_tiles_s ? p.rts[p.W + 2] : p.n_tiles_s;
  const unsigned ne = p.rte[p.W + 2] < p.n_tiles_e ? p.rte[p.W + 2] : p.n_tiles_e;
  unsigned bad = 0;
  for (unsigned i = blockIdx.x * blockDim.x + threadIdx.x; i < ns + ne; i += gridDim.x * blockDim.x) {
    const bool smp = i < ns;
    const TileMeta *meta = smp ? p.smeta : p.emeta;
    const unsigned t = smp ? i : i - ns;
    const TileMeta m = meta[t];
    bool b = (m.flags & 2u) != 0;
    if ((m.flags & 1u) && !b)
      for (unsigned j = t; j-- > 0;) {
        const TileMeta q = meta[j];
        if (q.flags & 1u) {
          b = m.first_ts < q.last_ts;
          break;
        }
      }
    if (b) bad |= smp ? 1u : 2u;
  }
  bad = __reduce_or_sync(kFull, bad);
  if ((threadIdx.x & 31) == 0 && bad) atomicOr(p.status, bad);
}

// ============================================================================================
// K5: top-k (Bottleneck Analyzer list).  One CTA per window.  Fullness key:
// key32 = 0xFFFFFFFF if level == cap else floor(level * 2^32 / cap), exactly order-preserving
// for cap <= 65535; size mode key32 = level.  MSB-first radix select (4 x 8
// bits) finds the k-th key tau; keys > tau are taken, keys == tau are taken in buffer_id order
// (tie-break), and the k winners are bitonic-sorted by (key desc, id asc).
// ============================================================================================
constexpr int kTopkThreads = 512;
constexpr unsigned kTopkCand = 4096;  // candidate list capacity after the first radix digit

// key32 = floor(l * 2^32 / c) for l < c, exact: m = floor(2^48 / c) (rcp table), q0 = (l*m) >> 16
// is floor or floor-1 (error < l / 2^16 < 1), one remainder test fixes it.
__device__ __forceinline__ unsigned fullness_key(unsigned l, unsigned c, int mode, const unsigned long long *rcp) {
  if (mode == RTM_RANK_SIZE) return l;
  if (l >= c) return 0xFFFFFFFFu;  // l == c for field-valid data
  unsigned long long q = ((unsigned long long)l * __ldg(rcp + c)) >> 16;
  const unsigned long long r = ((unsigned long long)l << 32) - q * c;
  if (r >= c) ++q;
  return (unsigned)q;
}

template <bool ALL>
__global__ void __launch_bounds__(kTopkThreads) k_topk(Params p) {
  extern __shared__ __align__(16) unsigned char smem[];
  const unsigned key_cap = ALL ? p.tk_slice_len : p.n_elig;  // keys one CTA ranks at most
  const bool keys_in_smem = key_cap <= kTopkSmemKeys;
  unsigned *keys = reinterpret_cast<unsigned *>(smem);                                  // [ne] or none
  unsigned *hist = keys + (keys_in_smem ? ((key_cap + 1) & ~1u) : 0);                        // [8][256]
  unsigned long long *sel = reinterpret_cast<unsigned long long *>(hist + 8 * 256);     // [1024]
  unsigned *cand = reinterpret_cast<unsigned *>(sel + 1024);                             // [kTopkCand]
  __shared__ unsigned scan_scratch[32];
  __shared__ unsigned s_digit, s_need, s_ngt, s_ncand;
  const unsigned w = blockIdx.x;
  const uint16_t *lv = p.lastlvl + (size_t)w * p.nb;
  const int warp = threadIdx.x >> 5;
  // few windows (streaming): the buffers of a window are split into id slices, one CTA each;
  // every slice keeps its own top-k candidates and k_topk_merge ranks their union (exact: the
  // global top-k is contained in the union of the slices' top-k)
  const unsigned slo = ALL ? blockIdx.y * p.tk_slice_len : 0u;
  const unsigned ne = ALL ? min(p.nb - slo, p.tk_slice_len) : p.n_elig;  // ranked buffers (ids ascending)
  auto id_of = [&](unsigned i) -> unsigned { return ALL ? slo + i : __ldg(p.elig_ids + i); };
  auto key_at = [&](unsigned i) -> unsigned {
    if (keys_in_smem) return keys[i];
    const unsigned b = id_of(i);
    return fullness_key(lv[b], __ldg(p.cap + b), p.rank_mode, p.rcp);
  };
  const unsigned keff = p.k < ne ? p.k : ne;
  const bool sliced = ALL && p.tk_slices > 1;
  unsigned long long *scr = sliced ? p.tk_scratch + ((size_t)w * p.tk_slices + blockIdx.y) * p.k : nullptr;
  if (keff == 0) {
    if (threadIdx.x == 0 && !sliced) p.topk_n[w] = 0;
    if (sliced)
      for (unsigned i = threadIdx.x; i < p.k; i += blockDim.x) scr[i] = 0ull;
    return;
  }
  // Full-prefix shortcut (Percent mode): a 100 %-full buffer has the largest possible key
  // (0xFFFFFFFF), so if the k lowest ids holding it are found while scanning in id order, they
  // ARE the top-k (ties by id) and the rest of the window is never read.  In the bottleneck
  // picture (L197-L199) that is a short prefix of the ids; otherwise the scan reaches the end
  // and the general path below runs.
  bool fast = false;
  if (p.rank_mode == RTM_RANK_PERCENT) {
    const bool vec = ALL && (p.nb & 7u) == 0;  // 8 consecutive buffers per thread (16-B loads)
    const unsigned per = vec ? 8u : 1u, step = blockDim.x * per;
    unsigned found = 0;
    for (unsigned base = 0; base < ne && found < keff; base += step) {
      const unsigned i0 = base + threadIdx.x * per;
      unsigned fm = 0;  // bit q: buffer i0 + q is 100 % full
      if (vec) {
        if (i0 < ne) {
          const uint4 L = reinterpret_cast<const uint4 *>(lv + slo)[i0 / 8];
          const uint4 C = __ldg(reinterpret_cast<const uint4 *>(p.cap + slo) + i0 / 8);
          const unsigned lw[4] = {L.x, L.y, L.z, L.w}, cw[4] = {C.x, C.y, C.z, C.w};
#pragma unroll
          for (int q = 0; q < 4; ++q) {
            fm |= ((lw[q] & 0xFFFFu) >= (cw[q] & 0xFFFFu) ? 1u : 0u) << (2 * q);
            fm |= ((lw[q] >> 16) >= (cw[q] >> 16) ? 1u : 0u) << (2 * q + 1);
          }
        }
      } else if (i0 < ne) {
        const unsigned b = id_of(i0);
        fm = lv[b] >= __ldg(p.cap + b) ? 1u : 0u;
      }
      unsigned tot;
      unsigned pos = found + block_excl_scan(__popc(fm), scan_scratch, &tot);
      for (unsigned x = fm; x && pos < keff; x &= x - 1, ++pos)
        sel[pos] = (0xFFFFFFFFull << 32) | (0xFFFFFFFFu - id_of(i0 + __ffs(x) - 1));
      found += tot;
    }
    fast = found >= keff;
  }
  bool top_tie = fast;  // winners share one key and were written in id order
  if (!fast) {
  // keys (shared memory when they fit) and, in the same pass, the largest key and how many
  // buffers hold it (per thread, then per warp, then per CTA)
  __shared__ unsigned s_max, s_cnt_max;
  if (threadIdx.x == 0) s_max = 0, s_cnt_max = 0;
  unsigned tm = 0, tc = 0;
  auto track = [&](unsigned k) {
    if (k > tm) tm = k, tc = 0;
    tc += (k == tm);
  };
  if (keys_in_smem && ALL && (p.nb & 7u) == 0) {  // 8 consecutive buffers per thread: 16-B loads
    const uint4 *lv4 = reinterpret_cast<const uint4 *>(lv + slo);  // slices start at multiples of 8
    const uint4 *cp4 = reinterpret_cast<const uint4 *>(p.cap + slo);
    uint4 *k4 = reinterpret_cast<uint4 *>(keys);
#pragma unroll 1  // unroll 2 spilled 12 B (ptxas) at the 128-register cap of 512 threads
    for (unsigned g = threadIdx.x; g < ne / 8; g += blockDim.x) {
      const uint4 L = lv4[g], C = __ldg(cp4 + g);
      const unsigned lw[4] = {L.x, L.y, L.z, L.w}, cw[4] = {C.x, C.y, C.z, C.w};
      unsigned kk[8];
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        kk[2 * q] = fullness_key(lw[q] & 0xFFFFu, cw[q] & 0xFFFFu, p.rank_mode, p.rcp);
        kk[2 * q + 1] = fullness_key(lw[q] >> 16, cw[q] >> 16, p.rank_mode, p.rcp);
      }
#pragma unroll
      for (int q = 0; q < 8; ++q) track(kk[q]);
      k4[2 * g] = make_uint4(kk[0], kk[1], kk[2], kk[3]);
      k4[2 * g + 1] = make_uint4(kk[4], kk[5], kk[6], kk[7]);
    }
  } else {
    for (unsigned i = threadIdx.x; i < ne; i += blockDim.x) {
      const unsigned b = id_of(i);
      const unsigned k = fullness_key(lv[b], __ldg(p.cap + b), p.rank_mode, p.rcp);
      if (keys_in_smem) keys[i] = k;
      track(k);
    }
  }
  {
    const unsigned wm = __reduce_max_sync(kFull, tm);
    const unsigned wc = __reduce_add_sync(kFull, tm == wm ? tc : 0u);
    __syncthreads();
    if ((threadIdx.x & 31) == 0) atomicMax(&s_max, wm);
    __syncthreads();
    if ((threadIdx.x & 31) == 0 && wm == s_max && wc) atomicAdd(&s_cnt_max, wc);
    __syncthreads();
  }
  // Shortcut: when the largest key is held by >= k buffers, the answer is the k lowest ids
  // holding it: tau = max key.
  top_tie = s_cnt_max >= keff;
  // MSB radix select.  After the first digit only candidates (top byte >= the selected digit,
  // at most k + the selected bucket) can matter: they are compacted in id order when they fit,
  // so the remaining passes and the selection scan ~1k keys instead of every buffer.
  unsigned prefix = top_tie ? s_max : 0u, mask = 0, need = keff;
  unsigned n_it = ne;  // iteration space: all keys, or the candidate list
  bool use_c = false;
  for (int d = top_tie ? -1 : 3; d >= 0; --d) {
    for (unsigned i = threadIdx.x; i < 8 * 256; i += blockDim.x) hist[i] = 0;
    __syncthreads();
    unsigned *myh = hist + (warp & 7) * 256;
    // warp-aggregated increments: many keys share a digit (empty / full buffers), and same-address
    // shared atomics serialise; __match_any_sync costs ~2 cycles per distinct digit in the warp
    const unsigned lane = threadIdx.x & 31;
    for (unsigned j0 = threadIdx.x - lane; j0 < n_it; j0 += blockDim.x) {
      const unsigned j = j0 + lane;
      bool ok = false;
      unsigned dg = 0;
      if (j < n_it) {
        const unsigned k = key_at(use_c ? cand[j] : j);
        ok = (k & mask) == prefix;
        dg = (k >> (8 * d)) & 255u;
      }
      const unsigned peers = __match_any_sync(kFull, ok ? dg : 0xFFFFFFFFu);
      if (ok && lane == (unsigned)__ffs(peers) - 1) atomicAdd(&myh[dg], (unsigned)__popc(peers));
    }
    __syncthreads();
    if (threadIdx.x < 256) {
      unsigned t = 0;
      for (int q = 0; q < 8; ++q) t += hist[q * 256 + threadIdx.x];
      hist[threadIdx.x] = t;  // row 0 <- totals (each thread owns its column)
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
      s_ncand = cum + hist[x];
    }
    __syncthreads();
    const unsigned digit = s_digit;
    if (d == 3 && s_ncand <= kTopkCand) {  // compact candidates (stable, id order)
      const unsigned chunk = (ne + blockDim.x - 1) / blockDim.x, c0 = threadIdx.x * chunk;
      unsigned cnt = 0;
      for (unsigned i = c0; i < c0 + chunk && i < ne; ++i) cnt += (key_at(i) >> 24) >= digit;
      unsigned pos = block_excl_scan(cnt, scan_scratch, nullptr);
      for (unsigned i = c0; i < c0 + chunk && i < ne; ++i)
        if ((key_at(i) >> 24) >= digit) cand[pos++] = i;
      n_it = s_ncand;
      use_c = true;
    }
    prefix |= digit << (8 * d);
    mask |= 255u << (8 * d);
    need = s_need;
    __syncthreads();
  }
  const unsigned tau = prefix;  // k-th key; `need` keys equal to tau are taken (lowest ids)
  if (threadIdx.x == 0) s_ngt = 0;
  __syncthreads();
  // one pass over contiguous chunks (id order): keys > tau (any order) and the first `need` == tau
  const unsigned chunk = (n_it + blockDim.x - 1) / blockDim.x;
  const unsigned c0 = threadIdx.x * chunk;
  unsigned ceq = 0;
  for (unsigned j = c0; j < c0 + chunk && j < n_it; ++j) {
    const unsigned i = use_c ? cand[j] : j;
    const unsigned k = key_at(i);
    if (k > tau) {
      const unsigned slot = atomicAdd(&s_ngt, 1u);
      sel[slot] = ((unsigned long long)k << 32) | (0xFFFFFFFFu - id_of(i));
    }
    ceq += (k == tau);
  }
  unsigned rank = block_excl_scan(ceq, scan_scratch, nullptr);  // syncs: s_ngt final after it
  const unsigned ngt = s_ngt;
  for (unsigned j = c0; j < c0 + chunk && j < n_it && rank < need; ++j) {
    const unsigned i = use_c ? cand[j] : j;
    const unsigned k = key_at(i);
    if (k == tau) {
      sel[ngt + rank] = ((unsigned long long)k << 32) | (0xFFFFFFFFu - id_of(i));
      ++rank;
    }
  }
  }  // general path
  __syncthreads();
  if (sliced) {  // this slice's candidates (unsorted); k_topk_merge ranks the union
    for (unsigned i = threadIdx.x; i < p.k; i += blockDim.x) scr[i] = i < keff ? sel[i] : 0ull;
    return;
  }
  // bitonic sort descending over the next power of two >= keff (top tie: the winners share one
  // key and were written in id order, so they are already sorted)
  unsigned P = 1;
  while (!top_tie && P < keff) P <<= 1;
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
      out = (unsigned long long)(p.gid ? __ldg(p.gid + b) : b) | ((unsigned long long)lv[b] << 32) |
            ((unsigned long long)__ldg(p.cap + b) << 48);
      if (p.persist_inline) atomicAdd(p.persist + (unsigned)(out & 0xFFFFFFFFull), 1u);  // k_persist fused
    }
    p.topk[(size_t)w * p.k + i] = out;
  }
  if (threadIdx.x == 0) p.topk_n[w] = keff;
}

// One CTA per window: the union of the slices' candidates (composite key32 << 32 | ~id, padding
// 0 ranks last) bitonic-sorted descending; the first min(k, nb) are the window's top-k.
constexpr unsigned kTopkMergeMax = 4096;
__global__ void __launch_bounds__(1024) k_topk_merge(Params p) {
  __shared__ unsigned long long v[kTopkMergeMax];
  const unsigned w = blockIdx.x;
  const unsigned n = p.tk_slices * p.k;
  unsigned P = 1;
  while (P < n) P <<= 1;
  const unsigned long long *src = p.tk_scratch + (size_t)w * n;
  for (unsigned i = threadIdx.x; i < P; i += blockDim.x) v[i] = i < n ? src[i] : 0ull;
  // slice 0 holds the lowest ids: if all its k candidates are 100 % full (the largest key) they
  // are the answer, already in id order (full-prefix shortcut of k_topk) - no sort
  bool full0 = true;
  for (unsigned i = threadIdx.x; i < (p.k < p.nb ? p.k : p.nb); i += blockDim.x)
    full0 &= (src[i] >> 32) == 0xFFFFFFFFull;
  if (__syncthreads_and(full0)) P = 1;
  for (unsigned size = 2; size <= P; size <<= 1) {
    for (unsigned stride = size >> 1; stride > 0; stride >>= 1) {
      for (unsigned i = threadIdx.x; i < P; i += blockDim.x) {
        const unsigned jx = i ^ stride;
        if (jx > i) {
          const bool desc = (i & size) == 0;
          const unsigned long long a = v[i], b = v[jx];
          if ((a < b) == desc) { v[i] = b; v[jx] = a; }
        }
      }
      __syncthreads();
    }
  }
  const unsigned keff = p.k < p.nb ? p.k : p.nb;
  const uint16_t *lv = p.lastlvl + (size_t)w * p.nb;
  for (unsigned i = threadIdx.x; i < p.k; i += blockDim.x) {
    unsigned long long out = 0xFFFFFFFFull;  // buffer_id 0xFFFFFFFF, level 0, cap 0
    if (i < keff) {
      const unsigned b = 0xFFFFFFFFu - (unsigned)(v[i] & 0xFFFFFFFFu);
      out = (unsigned long long)(p.gid ? __ldg(p.gid + b) : b) | ((unsigned long long)lv[b] << 32) |
            ((unsigned long long)__ldg(p.cap + b) << 48);
      if (p.persist_inline) atomicAdd(p.persist + (unsigned)(out & 0xFFFFFFFFull), 1u);  // k_persist fused
    }
    p.topk[(size_t)w * p.k + i] = out;
  }
  if (threadIdx.x == 0) p.topk_n[w] = keff;
}

// K5 for rank mode MEAN: one CTA per window over the 64-bit keys of the fold (mean_key).  MSB
// radix select over 8 x 8-bit digits (keys read from L2; windows shorter than 2^32 ticks leave the
// top bytes zero, one pass each); as soon as the keys at or above the selected prefix fit the
// candidate list they are compacted in id order and the remaining digits scan only them.  Keys >
// tau are taken, then the first `need` keys == tau in id order; the k winners are bitonic-sorted by
// (key desc, id asc).
constexpr int kT64Threads = 512;
constexpr unsigned kT64Cand = 8192;
__global__ void __launch_bounds__(kT64Threads) k_topk64(Params p) {
  __shared__ unsigned hist[256];
  __shared__ unsigned scan_scratch[32];
  __shared__ unsigned s_digit, s_need, s_ncand, s_ngt;
  __shared__ unsigned cand[kT64Cand];
  __shared__ unsigned long long selk[1024];
  __shared__ unsigned seli[1024];
  // candidates: the eligible buffers (owned components; all when n_elig == nb), indexed in id order
  const bool sub = p.n_elig < p.nb;
  const unsigned w = blockIdx.x, ne = sub ? p.n_elig : p.nb, lane = threadIdx.x & 31;
  const unsigned long long *keyw = p.mkey + (size_t)w * p.nb;
  auto K = [&](unsigned i) { return __ldcg(keyw + (sub ? __ldg(p.elig_ids + i) : i)); };
  const unsigned keff = p.k < ne ? p.k : ne;
  unsigned long long prefix = 0, mask = 0;
  unsigned need = keff, n_it = ne;
  bool use_c = false;
  for (int d = 7; d >= 0; --d) {
    for (unsigned i = threadIdx.x; i < 256; i += blockDim.x) hist[i] = 0;
    __syncthreads();
    for (unsigned j0 = threadIdx.x - lane; j0 < n_it; j0 += blockDim.x) {
      const unsigned j = j0 + lane;
      bool ok = false;
      unsigned dg = 0;
      if (j < n_it) {
        const unsigned long long k = K(use_c ? cand[j] : j);
        ok = (k & mask) == prefix;
        dg = (unsigned)(k >> (8 * d)) & 255u;
      }
      const unsigned peers = __match_any_sync(kFull, ok ? dg : 0xFFFFFFFFu);
      if (ok && lane == (unsigned)__ffs(peers) - 1) atomicAdd(&hist[dg], (unsigned)__popc(peers));
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
      s_ncand = (keff - need) + cum + hist[x];  // keys at or above the new prefix
    }
    __syncthreads();
    prefix |= (unsigned long long)s_digit << (8 * d);
    mask |= 255ull << (8 * d);
    if (!use_c && d > 0 && s_ncand <= kT64Cand) {  // compact keys >= the prefix, id order
      const unsigned long long lim = prefix >> (8 * d);
      const unsigned chunk = (ne + blockDim.x - 1) / blockDim.x, c0 = threadIdx.x * chunk;
      unsigned cnt = 0;
      for (unsigned i = c0; i < c0 + chunk && i < ne; ++i) cnt += (K(i) >> (8 * d)) >= lim;
      unsigned pos = block_excl_scan(cnt, scan_scratch, nullptr);
      for (unsigned i = c0; i < c0 + chunk && i < ne; ++i)
        if ((K(i) >> (8 * d)) >= lim) cand[pos++] = i;
      n_it = s_ncand;
      use_c = true;
    }
    need = s_need;
    __syncthreads();
  }
  const unsigned long long tau = prefix;
  if (threadIdx.x == 0) s_ngt = 0;
  __syncthreads();
  const unsigned chunk = (n_it + blockDim.x - 1) / blockDim.x, c0 = threadIdx.x * chunk;
  unsigned ceq = 0;
  for (unsigned j = c0; j < c0 + chunk && j < n_it; ++j) {
    const unsigned i = use_c ? cand[j] : j;
    const unsigned long long k = K(i);
    if (k > tau) {
      const unsigned slot = atomicAdd(&s_ngt, 1u);
      selk[slot] = k;
      seli[slot] = i;
    }
    ceq += (k == tau);
  }
  unsigned rank = block_excl_scan(ceq, scan_scratch, nullptr);
  const unsigned ngt = s_ngt;
  for (unsigned j = c0; j < c0 + chunk && j < n_it && rank < need; ++j) {
    const unsigned i = use_c ? cand[j] : j;
    if (K(i) == tau) {
      selk[ngt + rank] = tau;
      seli[ngt + rank] = i;
      ++rank;
    }
  }
  __syncthreads();
  unsigned P = 1;
  while (P < keff) P <<= 1;
  for (unsigned i = keff + threadIdx.x; i < P; i += blockDim.x) selk[i] = 0ull, seli[i] = 0xFFFFFFFFu;
  __syncthreads();
  for (unsigned size = 2; size <= P; size <<= 1) {  // (key desc, id asc)
    for (unsigned stride = size >> 1; stride > 0; stride >>= 1) {
      for (unsigned i = threadIdx.x; i < P; i += blockDim.x) {
        const unsigned jx = i ^ stride;
        if (jx > i) {
          const bool desc = (i & size) == 0;
          const unsigned long long a = selk[i], b = selk[jx];
          const unsigned ia = seli[i], ib = seli[jx];
          const bool a_before_b = a > b || (a == b && ia < ib);
          if (a_before_b != desc) {
            selk[i] = b; selk[jx] = a;
            seli[i] = ib; seli[jx] = ia;
          }
        }
      }
      __syncthreads();
    }
  }
  const uint16_t *lv = p.lastlvl + (size_t)w * p.nb;
  for (unsigned i = threadIdx.x; i < p.k; i += blockDim.x) {
    unsigned long long out = 0xFFFFFFFFull;
    if (i < keff) {
      const unsigned b = sub ? __ldg(p.elig_ids + seli[i]) : seli[i];
      out = (unsigned long long)(p.gid ? __ldg(p.gid + b) : b) | ((unsigned long long)lv[b] << 32) |
            ((unsigned long long)__ldg(p.cap + b) << 48);
      if (p.persist_inline) atomicAdd(p.persist + (unsigned)(out & 0xFFFFFFFFull), 1u);  // k_persist fused
    }
    p.topk[(size_t)w * p.k + i] = out;
    if (p.tkey) p.tkey[(size_t)w * p.k + i] = i < keff ? selk[i] : 0ull;  // world > 1: for the merge
  }
  if (threadIdx.x == 0) p.topk_n[w] = keff;
}

// Windows-in-top-k counter: one thread per (window, rank) of the call's (merged) lists.
__global__ void k_persist(Params p) {
  const size_t t = (size_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (t >= (size_t)p.W * p.k) return;
  const unsigned w = (unsigned)(t / p.k), i = (unsigned)(t % p.k);
  if (i < p.topk_n[w]) atomicAdd(p.persist + (unsigned)(p.topk[t] & 0xFFFFFFFFull), 1u);
}

// ============================================================================================
// K6: hang flag (L227-L229): cond_c(w) = any buffer of c full for the whole window AND no task
// event of c in w; run_c counts consecutive cond windows; flagged when run_c >= H.
// run_c(w) >= H  <=>  cond_c holds in windows w-H+1..w (reaching back into the carried run_in
// when w < H-1), so every (window, 32-component word) is flagged independently with bitwise ANDs.
// Threads [W*ncw, W*ncw + nc) compute the carried run length for the next call.
// ============================================================================================
__device__ __forceinline__ unsigned hang_cond(const Params &p, unsigned j, unsigned q) {
  const size_t i = (size_t)j * p.ncw + q;
  return __ldg(p.anyfull + i) & ~__ldg(p.active + i);
}

// Long H (> kHangShortH): the per-(window, word) AND loop costs O(run length) per thread and
// runs are long when components stay quiet (C5: H = 2048), so one thread per word computes the
// sliding-window AND over H windows in two passes (van Herk / Gil-Werman): prefix ANDs inside
// blocks of H windows forward, suffix ANDs backward; the range [w-H+1, w] is suffix(w-H+1) &
// prefix(w).  Windows w < H-1 reach before the call: prefix(w) (= AND over 0..w) and the carried
// run must cover the rest.
constexpr unsigned kHangShortH = 64;
// calls shorter than H with a long H (C5: 1000-window calls, H = 2048) take k_hang_prefix
__host__ __device__ constexpr bool hang_prefix_path(uint32_t W, uint32_t H) { return H > kHangShortH && W < H; }
__host__ __device__ constexpr size_t hang_flag_threads(uint32_t W, uint32_t ncw, uint32_t H) {
  return hang_prefix_path(W, H) ? 0 : H > kHangShortH ? (size_t)ncw : (size_t)W * ncw;
}

// Long H and a call shorter than H: every window w of the call is flagged iff the condition held
// in windows 0..w of the call (a prefix AND) and the carried run covers the rest (run_in >= H-1-w).
// One warp per 32-component word, lane = window inside a group of 32: the prefix AND is a warp
// scan, the carried-run test a per-bit threshold (first window at which the bit may be flagged).
__global__ void __launch_bounds__(256) k_hang_prefix(Params p) {
  const unsigned q = (unsigned)(((size_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5), lane = threadIdx.x & 31;
  if (q >= p.ncw) return;  // warp-uniform
  const unsigned H = p.H, W = p.W;
  const unsigned vmask = (q == p.ncw - 1 && (p.nc & 31)) ? (1u << (p.nc & 31)) - 1u : 0xFFFFFFFFu;
  // lane b: the first window of the call at which component q*32+b may be flagged
  const unsigned cc = q * 32 + lane;
  const unsigned r = cc < p.nc ? p.run[cc] : 0u;
  const unsigned first_ok_lane = r >= H - 1 ? 0u : H - 1 - r;
  unsigned acc = 0xFFFFFFFFu;  // AND of the condition over the windows before this group
  for (unsigned w0 = 0; w0 < W && __any_sync(kFull, acc != 0); w0 += 32) {
    const unsigned w = w0 + lane;
    unsigned x = w < W ? hang_cond(p, w, q) : 0xFFFFFFFFu;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {  // inclusive prefix AND over the group's windows
      const unsigned y = __shfl_up_sync(kFull, x, o);
      if (lane >= (unsigned)o) x &= y;
    }
    x &= acc;
    acc = __shfl_sync(kFull, x, 31);
    // bits whose carried run already covers window w (thresholds gathered from their lanes)
    unsigned elig = 0;
#pragma unroll
    for (int b = 0; b < 32; ++b) elig |= (w >= (unsigned)__shfl_sync(kFull, first_ok_lane, b) ? 1u : 0u) << b;
    const unsigned out = x & elig & vmask;
    if (w < W) {
      p.hung[(size_t)w * p.ncw + q] = out;
      if (out) atomicAdd(p.win + WF_HUNG * p.W + w, (unsigned long long)__popc(out));
    }
  }
  // windows after the prefix AND emptied: nothing flagged (hung rows are cleared per call)
}

// Long H, calls of >= H windows (C4: H = 96, 2000 windows): the van Herk passes of k_hang run
// block-parallel instead of one thread per word walking every window.  Pass 1, one thread per
// (word, block of H windows): prefix ANDs into hung[w], suffix ANDs into hsfx[w].  Pass 2, one
// thread per (window, word): hung[w] = hsfx[w - H + 1] & prefix(w) for w >= H - 1, the carried
// run for the windows before (C4: 1.66 ms -> 0.16 ms; the one-thread-per-word walk ran 8192
// threads over 2000 dependent windows).
__global__ void __launch_bounds__(256) k_hang_blocks(Params p) {
  const size_t tid = (size_t)blockIdx.x * blockDim.x + threadIdx.x;
  const unsigned nblk = (p.W + p.H - 1) / p.H;
  if (tid >= (size_t)nblk * p.ncw) return;
  const unsigned q = (unsigned)(tid % p.ncw), k = (unsigned)(tid / p.ncw);
  const unsigned w0 = k * p.H, w1 = min(p.W, w0 + p.H);
  unsigned acc = 0xFFFFFFFFu;
  for (unsigned w = w0; w < w1; ++w) {
    acc &= hang_cond(p, w, q);
    p.hung[(size_t)w * p.ncw + q] = acc;
  }
  unsigned suf = 0xFFFFFFFFu;
  for (unsigned w = w1; w-- > w0;) {
    suf &= hang_cond(p, w, q);
    p.hsfx[(size_t)w * p.ncw + q] = suf;
  }
}

__global__ void __launch_bounds__(256) k_hang_combine(Params p) {
  const size_t tid = (size_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (tid >= (size_t)p.W * p.ncw) return;
  const unsigned w = (unsigned)(tid / p.ncw), q = (unsigned)(tid % p.ncw), H = p.H;
  const unsigned vmask = (q == p.ncw - 1 && (p.nc & 31)) ? (1u << (p.nc & 31)) - 1u : 0xFFFFFFFFu;
  const unsigned pre = p.hung[tid];  // AND over [block start, w]
  unsigned out;
  if (w + 1 >= H) {
    out = __ldcg(p.hsfx + (size_t)(w + 1 - H) * p.ncw + q) & pre & vmask;
  } else {  // windows 0 .. H-2 (block 0's prefix): the carried run must cover the rest
    unsigned elig = 0;
    for (unsigned x = pre; x; x &= x - 1) {
      const unsigned b = __ffs(x) - 1, c = q * 32 + b;
      if (c < p.nc && p.run[c] >= H - 1 - w) elig |= 1u << b;
    }
    out = pre & elig & vmask;
  }
  p.hung[tid] = out;
  if (out) atomicAdd(p.win + WF_HUNG * p.W + w, (unsigned long long)__popc(out));
}

__global__ void k_hang(Params p) {
  const size_t tid = (size_t)blockIdx.x * blockDim.x + threadIdx.x;
  const bool lng = p.H > kHangShortH;
  const size_t nflag = p.hsfx ? 0 : hang_flag_threads(p.W, p.ncw, p.H);
  const size_t nflag_w = (nflag + 31) & ~(size_t)31;  // warp-aligned start of the run part
  if (lng && tid < nflag) {
    const unsigned q = (unsigned)tid, H = p.H, W = p.W;
    const unsigned vmask = (q == p.ncw - 1 && (p.nc & 31)) ? (1u << (p.nc & 31)) - 1u : 0xFFFFFFFFu;
    // window from which each component's carried run completes H (windows w < H-1 only)
    unsigned first_ok[32];
#pragma unroll
    for (int b = 0; b < 32; ++b) {
      const unsigned cc = q * 32 + b;
      const unsigned r = cc < p.nc ? p.run[cc] : 0u;
      first_ok[b] = r >= H - 1 ? 0u : H - 1 - r;
    }
    unsigned acc = 0;
    constexpr unsigned kB = 8;  // cond words loaded per batch (independent loads in flight)
    for (unsigned w0 = 0; w0 < W; w0 += kB) {  // forward: prefix AND inside blocks of H windows
      unsigned cb[kB];
#pragma unroll
      for (unsigned i = 0; i < kB; ++i) cb[i] = w0 + i < W ? hang_cond(p, w0 + i, q) : 0u;
#pragma unroll
      for (unsigned i = 0; i < kB; ++i) {
        const unsigned w = w0 + i;
        if (w >= W) break;
        acc = (w % H == 0) ? cb[i] : (acc & cb[i]);
        unsigned out = acc;
        if (w + 1 < H) {  // final here: needs the carried run (run_in >= H - (w+1))
          unsigned elig = 0;
          for (unsigned x = acc; x; x &= x - 1) {
            const unsigned b = __ffs(x) - 1;
            if (w >= first_ok[b]) elig |= 1u << b;
          }
          out = acc & elig & vmask;
          if (out) atomicAdd(p.win + WF_HUNG * p.W + w, (unsigned long long)__popc(out));
        }
        p.hung[(size_t)w * p.ncw + q] = out;  // w >= H-1: prefix(w), finished by the backward pass
      }
    }
    unsigned suf = 0;
    // backward: suffix AND inside blocks; only needed when some window of the call is >= H-1
    for (long long s0 = (long long)W - 1; W >= H && s0 >= 0; s0 -= kB) {
      unsigned cb[kB];
#pragma unroll
      for (unsigned i = 0; i < kB; ++i) cb[i] = s0 - (long long)i >= 0 ? hang_cond(p, (unsigned)(s0 - i), q) : 0u;
#pragma unroll
      for (unsigned i = 0; i < kB; ++i) {
        const long long s = s0 - (long long)i;
        if (s < 0) break;
        suf = ((unsigned long long)s % H == H - 1 || s == (long long)W - 1) ? cb[i] : (suf & cb[i]);
        const unsigned long long w = (unsigned long long)s + H - 1;
        if (w < W) {
          const unsigned f = suf & p.hung[(size_t)w * p.ncw + q] & vmask;
          p.hung[(size_t)w * p.ncw + q] = f;
          if (f) atomicAdd(p.win + WF_HUNG * p.W + w, (unsigned long long)__popc(f));
        }
      }
    }
  } else if (!lng && tid < nflag) {
    const unsigned w = (unsigned)(tid / p.ncw), q = (unsigned)(tid % p.ncw);
    const long long first = (long long)w - (long long)p.H + 1;
    unsigned acc = 0xFFFFFFFFu;
    for (long long j = w; j >= (first > 0 ? first : 0) && acc; --j) acc &= hang_cond(p, (unsigned)j, q);
    if (acc && first < 0) {  // the run must continue the carried run: run_in >= H - (w+1)
      const unsigned need = p.H - (w + 1);
      unsigned m = 0;
      for (unsigned x = acc; x; x &= x - 1) {
        const unsigned bit = __ffs(x) - 1, c = q * 32 + bit;
        if (c < p.nc && p.run[c] >= need) m |= 1u << bit;
      }
      acc = m;
    }
    if (q == p.ncw - 1 && (p.nc & 31)) acc &= (1u << (p.nc & 31)) - 1u;
    p.hung[(size_t)w * p.ncw + q] = acc;
    if (acc) atomicAdd(p.win + WF_HUNG * p.W + w, (unsigned long long)__popc(acc));
  } else if (tid >= nflag_w && tid < nflag_w + (size_t)p.ncw * 32) {
    // carried run length for the next call: one warp per 32-component word, lane = component.
    // Windows are taken 32 at a time from the last one backwards (lane l: window W-1-32g-l); one
    // ballot per component marks the windows where its condition fails, the first such lane ends
    // its run.  A run through every window of the call continues the carried run.
    const unsigned q = (unsigned)((tid - nflag_w) >> 5), lane = threadIdx.x & 31, c = q * 32 + lane;
    unsigned r = 0;
    bool done = false;
    for (unsigned g = 0; __any_sync(kFull, !done); ++g) {
      const long long j = (long long)p.W - 1 - 32ll * g - lane;
      const unsigned word = j >= 0 ? hang_cond(p, (unsigned)j, q) : 0xFFFFFFFFu;
      unsigned zeros = 0;  // this lane's component: windows of the group where cond fails
#pragma unroll 4
      for (unsigned b = 0; b < 32; ++b) {
        const unsigned m = __ballot_sync(kFull, j >= 0 && !((word >> b) & 1u));
        if (lane == b) zeros = m;
      }
      if (!done) {
        const long long left = (long long)p.W - 32ll * g;  // windows of the call not yet scanned
        if (zeros) {
          r += __ffs(zeros) - 1;
          done = true;
        } else if (left <= 32) {
          r += (unsigned)left + (c < p.nc ? p.run[c] : 0u);
          done = true;
        } else {
          r += 32;
        }
      }
    }
    if (c < p.nc) p.run_out[c] = r;
  }
}

// ============================================================================================
// K7: progress bars (L131): per kernel, cumulative START/END over windows (block scan), and
// the per-component cumulative counts for the last window.
// ============================================================================================
__global__ void __launch_bounds__(1024) k_progress(Params p) {
  __shared__ unsigned scan_scratch[32];
  const unsigned k = blockIdx.x;
  if (k < p.nk) {
    long long s = p.kstart[k], e = p.kend[k];
    const bool live = p.klive[k] != 0;  // a free bar id reads all zero (its counts stay zero)
    const long long total = live ? p.ktotal[k] : 0;
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
        o[1] = live ? S : 0;
        o[2] = live ? E : 0;
        o[3] = live ? S - E : 0;
        o[4] = live ? total - S : 0;
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
      p.cdelta[2 * c] = p.cdelta[2 * c + 1] = 0;  // consumed: zero for the next call
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
//   hung [W][ncw] u32 (padded) | comps [nc] (3 x i64) | bstat [pack_nb] (32 B; reserved = owned) |
//   gids [pack_nb] u32 (rank-local numbering only: the global id of each bstat entry, ~0 = pad) |
//   tkey [W][k] u64 (rank mode MEAN only: the order key of each top-k entry, mean_key)
// ============================================================================================
// Per-call exchange pack (world > 1): only what the per-window merged results need.
//   win   [kWinFields][W] u64   counters and digest (sums over ranks)
//   topk  [W][k] u64            local top-k entries (id | level << 32 | cap << 48)
//   topk_n[W] u32
//   kd    [W][nk][2] u32        this rank's START / END events per window and bar (the merge
//                               sums them and carries the merged cumulative counts across calls)
//   tkey  [W][k] u64            rank mode MEAN: each candidate's 64-bit order key
// The per-buffer table, per-component totals and hang bitmaps are NOT in it: they are exchanged on
// demand (rtm_tables_local / rtm_tables_merge / rtm_sync_tables).
struct PackLayout {
  size_t win, topk, topk_n, kd, tkey, total;
};
__host__ __device__ inline size_t align8(size_t x) { return (x + 7) & ~(size_t)7; }
__host__ __device__ inline PackLayout pack_layout_for(uint32_t W, uint32_t k, uint32_t nk, int rank_mode) {
  PackLayout L;
  size_t o = 0;
  L.win = o; o += align8((size_t)kWinFields * W * 8);
  L.topk = o; o += align8((size_t)W * k * 8);
  L.topk_n = o; o += align8((size_t)W * 4);
  L.kd = o; o += align8((size_t)W * nk * 2 * 4);
  L.tkey = o; o += rank_mode == RTM_RANK_MEAN ? (size_t)W * k * 8 : 0;
  L.total = o;
  return L;
}
__host__ __device__ inline PackLayout pack_layout(const Params &p) { return pack_layout_for(p.W, p.k, p.nk, p.rank_mode); }

// On-demand tables pack (the last call's state): per-component START / END totals, the
// per-buffer table of the last window (with global ids under a rank-local numbering) and the
// per-window hang bitmaps.
struct TablesLayout {
  size_t comps, bstat, gids, hung, total;
};
__host__ __device__ inline TablesLayout tables_layout(const Params &p) {
  TablesLayout L;
  size_t o = 0;
  L.comps = o; o += align8((size_t)p.nc * 16);
  L.bstat = o; o += align8((size_t)p.pack_nb * sizeof(rtm_buffer_stat));
  L.gids = o; o += p.gid ? align8((size_t)p.pack_nb * 4) : 0;
  L.hung = o; o += align8((size_t)p.W * p.ncw * 4);
  L.total = o;
  return L;
}

__device__ __forceinline__ unsigned long long topk_composite(unsigned long long ent, int mode,
                                                             const unsigned long long *rcp) {
  const unsigned b = (unsigned)(ent & 0xFFFFFFFFu);
  const unsigned l = (unsigned)(ent >> 32) & 0xFFFFu, c = (unsigned)(ent >> 48);
  return ((unsigned long long)fullness_key(l, c, mode, rcp) << 32) | (0xFFFFFFFFu - b);
}

// one CTA per window: merge world x k candidates; sums of scalar fields; progress sums; hang OR.
// Candidates rank by (key, sec) descending: PERCENT / SIZE key = fullness32 << 32 | ~id, sec = 0;
// MEAN key = the 64-bit mean_key from the pack, sec = ~id.  Padding (0, 0) ranks last: a real
// candidate has key >= 1 (PERCENT / SIZE) or sec >= 1 (MEAN, ids < 2^32 - 1).
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
  unsigned *sec = reinterpret_cast<unsigned *>(full_ent + P);  // [P] tie-break word (MEAN: ~id)
  const bool mean = p.rank_mode == RTM_RANK_MEAN;
  for (unsigned i = threadIdx.x; i < P; i += blockDim.x) {
    unsigned long long key = 0, en = 0;
    unsigned sc = 0;
    if (i < nc_all) {
      const unsigned r = i / p.k, s = i % p.k;
      const unsigned char *base = g + stride * r;
      const unsigned n = reinterpret_cast<const unsigned *>(base + L.topk_n)[w];
      if (s < n) {
        en = reinterpret_cast<const unsigned long long *>(base + L.topk)[(size_t)w * p.k + s];
        if (mean) {
          key = reinterpret_cast<const unsigned long long *>(base + L.tkey)[(size_t)w * p.k + s];
          sc = 0xFFFFFFFFu - (unsigned)(en & 0xFFFFFFFFull);
        } else {
          key = topk_composite(en, p.rank_mode, p.rcp);
        }
      }
    }
    cand[i] = key;
    full_ent[i] = en;
    sec[i] = sc;
  }
  __syncthreads();
  for (unsigned size = 2; size <= P; size <<= 1) {
    for (unsigned stride2 = size >> 1; stride2 > 0; stride2 >>= 1) {
      for (unsigned i = threadIdx.x; i < P; i += blockDim.x) {
        unsigned jx = i ^ stride2;
        if (jx > i) {
          bool desc = (i & size) == 0;
          unsigned long long a = cand[i], b = cand[jx];
          const unsigned sa = sec[i], sb = sec[jx];
          if ((a < b || (a == b && sa < sb)) == desc) {
            cand[i] = b; cand[jx] = a;
            sec[i] = sb; sec[jx] = sa;
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
}

// Merged progress bars (L131): one CTA per bar; the bar's START / END deltas summed over ranks,
// prefix-summed over the call's windows on top of the merged cumulative counts of earlier calls
// (gcum, identical on every rank), which are then advanced.
__global__ void __launch_bounds__(1024) k_merge_progress(Params p, const unsigned char *g, unsigned world,
                                                         size_t stride, long long *gcum) {
  __shared__ unsigned scan_scratch[32];
  const PackLayout L = pack_layout(p);
  const unsigned k = blockIdx.x;
  long long s = gcum[2 * k], e = gcum[2 * k + 1];
  const bool live = p.klive[k] != 0;  // a destroyed bar reads all zero (rtm_bar_destroy)
  const long long total = live ? p.ktotal[k] : 0;
  for (unsigned base = 0; base < p.W; base += blockDim.x) {
    const unsigned w = base + threadIdx.x;
    unsigned ds = 0, de = 0;
    if (w < p.W)
      for (unsigned r = 0; r < world; ++r) {
        const unsigned *kd = reinterpret_cast<const unsigned *>(g + stride * r + L.kd) + ((size_t)w * p.nk + k) * 2;
        ds += kd[0];
        de += kd[1];
      }
    unsigned ts_, te_;
    const unsigned xs = block_excl_scan(ds, scan_scratch, &ts_);
    const unsigned xe = block_excl_scan(de, scan_scratch, &te_);
    if (w < p.W) {
      const long long S = s + xs + ds, E = e + xe + de;
      long long *o = p.prog + ((size_t)w * p.nk + k) * 5;
      o[0] = total;
      o[1] = live ? S : 0;
      o[2] = live ? E : 0;
      o[3] = live ? S - E : 0;
      o[4] = live ? total - S : 0;
    }
    s += ts_;
    e += te_;
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    gcum[2 * k] = s;
    gcum[2 * k + 1] = e;
  }
}

__global__ void k_merge_tables(Params p, const unsigned char *g, unsigned world, size_t stride) {
  const TablesLayout L = tables_layout(p);
  const size_t tid = (size_t)blockIdx.x * blockDim.x + threadIdx.x, nth = (size_t)gridDim.x * blockDim.x;
  for (size_t c = tid; c < p.nc; c += nth) {
    rtm_component_tasks t = {0, 0, 0};
    for (unsigned r = 0; r < world; ++r) {
      const long long *x = reinterpret_cast<const long long *>(g + stride * r + L.comps) + 2 * c;
      t.started += x[0];
      t.finished += x[1];
    }
    t.in_flight = t.started - t.finished;
    p.comps[c] = t;
  }
  for (size_t q = tid; q < (size_t)p.W * p.ncw; q += nth) {  // hang flags: OR over ranks
    unsigned x = 0;
    for (unsigned r = 0; r < world; ++r) x |= reinterpret_cast<const unsigned *>(g + stride * r + L.hung)[q];
    p.hung[q] = x;
  }
  if (p.gid) {  // rank-local numbering: scatter every rank's entries to their global ids
    for (size_t q = tid; q < (size_t)world * p.pack_nb; q += nth) {
      const unsigned r = (unsigned)(q / p.pack_nb), i = (unsigned)(q % p.pack_nb);
      const unsigned gb = reinterpret_cast<const unsigned *>(g + stride * r + L.gids)[i];
      if (gb < p.n_global) p.bstat_g[gb] = reinterpret_cast<const rtm_buffer_stat *>(g + stride * r + L.bstat)[i];
    }
    return;
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

// this rank's tables pack
__global__ void k_pack_tables(Params p, unsigned char *d) {
  const TablesLayout L = tables_layout(p);
  const size_t tid = (size_t)blockIdx.x * blockDim.x + threadIdx.x, nth = (size_t)gridDim.x * blockDim.x;
  for (size_t c = tid; c < p.nc; c += nth) {
    long long *x = reinterpret_cast<long long *>(d + L.comps) + 2 * c;
    x[0] = p.cstart[c];
    x[1] = p.cend[c];
  }
}

// world == 1 with a rank-local numbering: the table by global id
__global__ void k_scatter_bstat(Params p) {
  for (size_t b = (size_t)blockIdx.x * blockDim.x + threadIdx.x; b < p.nb; b += (size_t)gridDim.x * blockDim.x)
    p.bstat_g[__ldg(p.gid + b)] = p.bstat[b];
}

#endif  // RTM_TU_PARTITION
}  // namespace

// ============================================================================================
// launchers
// ============================================================================================
constexpr uint32_t kTwoPassMinBins = 1024;
#ifdef RTM_TU_PARTITION
extern std::atomic<unsigned long long> g_kernel_launches;
inline void count_launch() { g_kernel_launches.fetch_add(1, std::memory_order_relaxed); }
#else
__global__ void k_clear(ClearList cl) { clear_ranges(cl); }

std::atomic<unsigned long long> g_kernel_launches{0};
inline void count_launch() { g_kernel_launches.fetch_add(1, std::memory_order_relaxed); }
unsigned long long kernel_launches() { return g_kernel_launches.load(std::memory_order_relaxed); }

void launch_clear(const ClearList &cl, cudaStream_t st) {
  if (!cl.n) return;
  unsigned long long mx = 0;
  for (int r = 0; r < cl.n; ++r) mx = cl.bytes[r] > mx ? cl.bytes[r] : mx;
  const unsigned blocks = (unsigned)((mx / 16 + 255) / 256 + 1);
  { k_clear<<<blocks < 1184 ? blocks : 1184, 256, 0, st>>>(cl); count_launch(); }
}

size_t fold_smem_bytes(int bin_log) {
  return (bin_log == 7 ? sizeof(FoldSmem<7>) : sizeof(FoldSmem<8>)) * kFoldWarps;
}
// measured (1 x B200, full-size configs): 320 bins (C3) the match-based partition and the two-pass
// path tie (28.5 vs 29.4 ms per step: k_subpart reads the entries twice at ~4 warp instructions
// each); 2560 bins (C5) fold 22.4 -> 17.9 ms per 10k windows; 4096 bins (C4) 132.5 -> 77.5 ms.
// Below it, 171 .. 1023 bins take the lane-major partition with multi-pass ranking (MP).
// lane-major partition: the capacity table in shared memory when two CTAs still fit per SM
bool partition_caps_smem(uint32_t nbins, uint32_t nb) { return k1_smem_lm(nbins, nb, true) + 1024 <= 113 * 1024; }
size_t partition_smem_bytes(uint32_t nbins, uint32_t nb) {
  return nbins < kTwoPassMinBins ? k1_smem_lm(nbins, nb, partition_caps_smem(nbins, nb)) : k1_smem_mx(nbins);
}
static_assert(2 * (k1_smem_lm(80, 20480) + 1024 + 512) <= 228 * 1024, "C2-sized partition CTAs must fit 2 per SM");
static_assert(k1_smem_lm(kLmMaxBins, 0, false) <= 113 * 1024 && k1_smem_lm(kTwoPassMinBins - 1, 0, false) <= 227 * 1024 &&
                  k1_smem_mx(kMaxBins) <= 227 * 1024,
              "partition shared memory exceeds the opt-in limit");
size_t topk_smem_bytes(uint32_t nb) {
  return (size_t)(nb <= kTopkSmemKeys ? ((nb + 1) & ~1u) : 0) * 4 + 8 * 256 * 4 + 1024 * 8 + kTopkCand * 4;
}

// Resident blocks per SM of a kernel at a block size / dynamic shared memory, cached per device:
// the occupancy query is a driver call of tens of microseconds, made on the launch path of every
// call otherwise (the GPU idled behind it between k_prep and the partition).
int occupancy(const void *fn, int threads, size_t smem) {
  struct Key {
    const void *fn;
    int threads, dev;
    size_t smem;
    bool operator<(const Key &o) const {
      return std::tie(fn, threads, dev, smem) < std::tie(o.fn, o.threads, o.dev, o.smem);
    }
  };
  static std::mutex mu;
  static std::map<Key, int> cache;
  int dev = 0;
  cudaGetDevice(&dev);
  const Key k{fn, threads, dev, smem};
  {
    std::lock_guard<std::mutex> g(mu);
    auto it = cache.find(k);
    if (it != cache.end()) return it->second;
  }
  int n = 0;
  if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n, fn, threads, smem) != cudaSuccess) {
    cudaGetLastError();
    n = 0;
  }
  if (n < 1) n = 1;
  std::lock_guard<std::mutex> g(mu);
  cache[k] = n;
  return n;
}

void launch_prep(const Params &p, const ClearList &cl, long long *Bs, long long *Be, int n_sms, cudaStream_t st) {
  static int per_sm[128] = {0};
  int dev = 0;
  cudaGetDevice(&dev);
  if (dev >= 0 && dev < 128 && !per_sm[dev]) {
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm[dev], k_prep, 256, 0);
    if (per_sm[dev] < 1) per_sm[dev] = 1;
  }
  const unsigned cap = (unsigned)(n_sms * per_sm[dev >= 0 && dev < 128 ? dev : 0]);
  unsigned long long mx = 0;
  for (int r = 0; r < cl.n; ++r) mx = cl.bytes[r] > mx ? cl.bytes[r] : mx;
  unsigned grid = (unsigned)std::max<unsigned long long>({(2ull * (p.W + 1) + 7) / 8, (mx / 16 + 255) / 256 + 1,
                                                          (unsigned long long)(p.W + 2), 2ull});
  if (grid > cap) grid = cap;
  // few-window calls (streaming): one block, block barriers instead of grid barriers
  if (p.W <= 4 && mx <= 64 * 1024) grid = 1;
  Params pp = p;
  ClearList cc = cl;
  void *args[] = {&pp, &cc, &Bs, &Be};
  cudaLaunchCooperativeKernel((const void *)k_prep, dim3(grid), dim3(256), args, 0, st);
  count_launch();
}

bool partition_two_pass(uint32_t nbins, bool narrow) { return nbins >= kTwoPassMinBins && narrow; }
bool partition_fuses_events(uint32_t nbins, uint32_t n_tiles_s, bool two_pass) {
  return n_tiles_s && (nbins < kTwoPassMinBins || two_pass);
}

template <int BL>
void launch_subpart_bl(const Params &p, int n_sms, cudaStream_t st) {
  const size_t sm = sizeof(SubSmem<BL>) * kSubWarps;
  const int per_sm = occupancy((const void *)k_subpart<BL>, kSubWarps * 32, sm);
  unsigned grid = (unsigned)(n_sms * per_sm);
  const unsigned need = (p.W * p.nsb + kSubWarps - 1) / kSubWarps;
  if (grid > need) grid = need;
  if (grid == 0) grid = 1;
  if (p.seq_ranges > 1u) { k_subpart<BL, true><<<grid, kSubWarps * 32, sm, st>>>(p); count_launch(); }
  else { k_subpart<BL><<<grid, kSubWarps * 32, sm, st>>>(p); count_launch(); }
}

void launch_subpart(const Params &p, int n_sms, cudaStream_t st) {
  if (!p.nsb || !p.n_tiles_s) return;
  if (p.bin_log == 7) launch_subpart_bl<7>(p, n_sms, st);
  else launch_subpart_bl<8>(p, n_sms, st);
}

void launch_events(const Params &p, cudaStream_t st) {
  if (!p.n_tiles_e) return;
  const size_t sm = (size_t)2 * p.nk * 4 + (p.ncw <= 2048 ? (size_t)p.ncw * 4 : 0);
  { k_events<<<p.n_tiles_e, kK3Threads, sm, st>>>(p); count_launch(); }
}

template <int BL>
void launch_fold_bl(const Params &p, int n_sms, cudaStream_t st) {
  const size_t sm = fold_smem_bytes(BL);
  const int per_sm = occupancy((const void *)k_fold<true, false, BL>, kFoldWarps * 32, sm);
  unsigned grid = (unsigned)(n_sms * per_sm);
  const unsigned units = p.W * p.nbins;
  const unsigned need = (units + kFoldWarps - 1) / kFoldWarps;
  if (grid > need) grid = need;
  if (grid == 0) grid = 1;
  // sparse: fewer than 2 samples per buffer and window on average (C3-C5 shapes), so many of a
  // unit's buffers are untouched and the look-back walks several windows
  const bool sparse = p.ns < 2ull * p.nb * p.W;
  // compacted finalize when fewer samples than buffer-windows (C4: 0.86, Zipf, ~40 % of a unit's
  // buffers touched: fold 31.8 -> 28.3 ms; C3 at 1.1 (2/3 touched) is faster without: 13.1 vs 15.9)
  const bool very_sparse = p.ns < 1ull * p.nb * p.W;
  if (p.narrow_d && very_sparse) { k_fold<true, true, BL, true, true><<<grid, kFoldWarps * 32, sm, st>>>(p); count_launch(); }
  else if (p.narrow_d && sparse) { k_fold<true, true, BL, false, true><<<grid, kFoldWarps * 32, sm, st>>>(p); count_launch(); }
  else if (p.narrow_d) { k_fold<true, false, BL, false, true><<<grid, kFoldWarps * 32, sm, st>>>(p); count_launch(); }
  else if (p.narrow && very_sparse) { k_fold<true, true, BL, true><<<grid, kFoldWarps * 32, sm, st>>>(p); count_launch(); }
  else if (p.narrow && sparse) { k_fold<true, true, BL><<<grid, kFoldWarps * 32, sm, st>>>(p); count_launch(); }
  else if (p.narrow) { k_fold<true, false, BL><<<grid, kFoldWarps * 32, sm, st>>>(p); count_launch(); }
  else if (sparse) { k_fold<false, true, BL><<<grid, kFoldWarps * 32, sm, st>>>(p); count_launch(); }
  else { k_fold<false, false, BL><<<grid, kFoldWarps * 32, sm, st>>>(p); count_launch(); }
}

// very sparse calls: fewer than 1 kept sample per 8 buffer-windows (C5 ~ 1 in 45); PERCENT / SIZE
bool fold_sequential(const Params &p) {
  return !p.mkey && p.W > 1 && (unsigned long long)p.ns * 8ull < (unsigned long long)p.nb * p.W;
}

template <int BL>
void launch_fold_seq(const Params &p, int n_sms, cudaStream_t st) {
  const size_t sm = sizeof(FoldSeqSmem<BL>) * kFoldWarps;
  const int per_sm = occupancy((const void *)k_fold_seq<true, BL>, kFoldWarps * 32, sm);
  unsigned grid = (unsigned)(n_sms * per_sm);
  const unsigned need = (p.nbins * (p.seq_ranges > 1u ? p.seq_ranges : 1u) + kFoldWarps - 1) / kFoldWarps;
  if (grid > need) grid = need;
  if (p.narrow_d) { k_fold_seq<true, BL, true><<<grid, kFoldWarps * 32, sm, st>>>(p); count_launch(); }
  else if (p.narrow) { k_fold_seq<true, BL><<<grid, kFoldWarps * 32, sm, st>>>(p); count_launch(); }
  else { k_fold_seq<false, BL><<<grid, kFoldWarps * 32, sm, st>>>(p); count_launch(); }
}

void launch_fold(const Params &p, int n_sms, cudaStream_t st) {
  if (fold_sequential(p)) {
    if (p.bin_log == 7) launch_fold_seq<7>(p, n_sms, st);
    else launch_fold_seq<8>(p, n_sms, st);
    return;
  }
  if (p.bin_log == 7) launch_fold_bl<7>(p, n_sms, st);
  else launch_fold_bl<8>(p, n_sms, st);
}

void launch_order_check(const Params &p, cudaStream_t st) {
  const unsigned n = p.n_tiles_s + p.n_tiles_e;  // upper bound; the kernel reads the device counts
  if (!n) return;
  unsigned blocks = (n + 255) / 256;
  blocks = blocks < 1184 ? blocks : 1184;
  { k_order_check<<<blocks, 256, 0, st>>>(p); count_launch(); }
}

uint32_t topk_slices(uint32_t nb, uint32_t k, uint32_t W, int n_sms, bool all, uint32_t *slice_len) {
  uint32_t P = 1;
  if (all && (nb & 7u) == 0 && W < (uint32_t)n_sms) {
    P = (2u * (uint32_t)n_sms + W - 1) / W;
    P = std::min(P, nb / 2048u);
    P = std::min(P, std::max(2u, 1024u / k));  // merge sorts <= max(1024, 2k) candidates
    if (P < 2) P = 1;
  }
  uint32_t L = P > 1 ? (((nb + P - 1) / P + 7) & ~7u) : nb;
  if (P > 1) P = (nb + L - 1) / L;
  *slice_len = L;
  return P;
}

void launch_topk(const Params &p, cudaStream_t st) {
  if (p.mkey) {  // rank mode MEAN
    { k_topk64<<<p.W, kT64Threads, 0, st>>>(p); count_launch(); }
    return;
  }
  if (p.n_elig == p.nb && p.tk_slices > 1) {
    { k_topk<true><<<dim3(p.W, p.tk_slices), kTopkThreads, topk_smem_bytes(p.tk_slice_len), st>>>(p); count_launch(); }
    { k_topk_merge<<<p.W, 1024, 0, st>>>(p); count_launch(); }
    return;
  }
  if (p.n_elig == p.nb) { k_topk<true><<<p.W, kTopkThreads, topk_smem_bytes(p.nb), st>>>(p); count_launch(); }
  else { k_topk<false><<<p.W, kTopkThreads, topk_smem_bytes(p.n_elig), st>>>(p); count_launch(); }
}

// Every host-side decision of rtm_window_reduce's launch sequence that is not a kernel argument
// (kernel variants, grid sizes, which kernels run): two calls with equal shapes on the same
// workspaces launch the same kernels with the same configurations, so a CUDA graph captured for
// one replays the other with only the Params argument replaced (rtm_api.cpp, rtm_use_graphs).
void launch_shape(const Params &p, uint64_t key[3]) {
  key[0] = (uint64_t)p.W | (uint64_t)p.n_tiles_s << 32;
  key[1] = (uint64_t)p.n_tiles_e | (uint64_t)p.tk_slices << 32;
  key[2] = (uint64_t)(p.narrow != 0) | (uint64_t)(p.fuse_events != 0) << 1 | (uint64_t)(p.nsb != 0) << 2 |
           (uint64_t)fold_sequential(p) << 3 | (uint64_t)(p.ns < 2ull * p.nb * p.W) << 4 |
           (uint64_t)(p.ns < 1ull * p.nb * p.W) << 11 | (uint64_t)(p.narrow_d != 0) << 12 |
           (uint64_t)(p.seq_ranges & 0xFu) << 20 | (uint64_t)(p.hsfx != nullptr) << 24 |
           (uint64_t)(p.mkey != nullptr) << 5 | (uint64_t)(p.n_elig == p.nb) << 6 |
           (uint64_t)hang_prefix_path(p.W, p.H) << 7 | (uint64_t)(p.n_tiles_s != 0) << 8 |
           (uint64_t)(p.n_tiles_e != 0) << 9 | (uint64_t)(p.t_inline != 0) << 10 | (uint64_t)p.bin_log << 16;
}
const void *prep_kernel_fn() { return (const void *)k_prep; }
void count_launches(unsigned n) { g_kernel_launches.fetch_add(n, std::memory_order_relaxed); }

void launch_persist(const Params &p, cudaStream_t st) {
  const size_t n = (size_t)p.W * p.k;
  if (!n || !p.persist) return;
  { k_persist<<<(unsigned)((n + 255) / 256), 256, 0, st>>>(p); count_launch(); }
}

bool hang_block_path(uint32_t W, uint32_t H) { return H > kHangShortH && W >= H; }  // k_hang_blocks + k_hang_combine

void launch_hang(const Params &p, cudaStream_t st) {
  const unsigned threads = 256;
  if (hang_prefix_path(p.W, p.H)) {
    const size_t nt = (size_t)p.ncw * 32;
    { k_hang_prefix<<<(unsigned)((nt + threads - 1) / threads), threads, 0, st>>>(p); count_launch(); }
  }
  if (p.hsfx) {  // long H, W >= H: block-parallel van Herk passes, then k_hang's carried runs only
    const size_t nb = (size_t)((p.W + p.H - 1) / p.H) * p.ncw, nw = (size_t)p.W * p.ncw;
    { k_hang_blocks<<<(unsigned)((nb + threads - 1) / threads), threads, 0, st>>>(p); count_launch(); }
    { k_hang_combine<<<(unsigned)((nw + threads - 1) / threads), threads, 0, st>>>(p); count_launch(); }
  }
  const size_t n = (p.hsfx ? 0 : ((hang_flag_threads(p.W, p.ncw, p.H) + 31) & ~(size_t)31)) + (size_t)p.ncw * 32;
  { k_hang<<<(unsigned)((n + threads - 1) / threads), threads, 0, st>>>(p); count_launch(); }
}

void launch_progress(const Params &p, cudaStream_t st) {
  // 1024 threads: one block scan covers up to 1024 windows per kernel bar (4 rounds at 256)
  const unsigned comp_blocks = (p.nc + 1023) / 1024 < 256 ? (p.nc + 1023) / 1024 : 256;
  { k_progress<<<p.nk + comp_blocks, 1024, 0, st>>>(p); count_launch(); }
}

uint64_t pack_bytes(const Params &p) { return pack_layout(p).total; }
uint64_t exchange_bytes(uint32_t W, uint32_t k, uint32_t nk, int rank_mode) {
  return pack_layout_for(W, k, nk, rank_mode).total;
}

void configure_kernels_once() {
  static bool done[128] = {false};
  int dev = 0;
  cudaGetDevice(&dev);
  if (dev < 0 || dev >= 128 || done[dev]) return;
  done[dev] = true;
  configure_partition_once();
  cudaFuncSetAttribute(k_subpart<7>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)(sizeof(SubSmem<7>) * kSubWarps));
  cudaFuncSetAttribute(k_subpart<8>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)(sizeof(SubSmem<8>) * kSubWarps));
  cudaFuncSetAttribute(k_subpart<7, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)(sizeof(SubSmem<7>) * kSubWarps));
  cudaFuncSetAttribute(k_subpart<8, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)(sizeof(SubSmem<8>) * kSubWarps));
  cudaFuncSetAttribute(k_topk<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)topk_smem_bytes(kTopkSmemKeys));
  cudaFuncSetAttribute(k_topk<false>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                       (int)topk_smem_bytes(kTopkSmemKeys));
#define RTM_FOLD_ATTR(NAR_, SP_, BL_) \
  cudaFuncSetAttribute(k_fold<NAR_, SP_, BL_>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)fold_smem_bytes(BL_))
  RTM_FOLD_ATTR(true, false, 8); RTM_FOLD_ATTR(false, false, 8); RTM_FOLD_ATTR(true, true, 8); RTM_FOLD_ATTR(false, true, 8);
  RTM_FOLD_ATTR(true, false, 7); RTM_FOLD_ATTR(false, false, 7); RTM_FOLD_ATTR(true, true, 7); RTM_FOLD_ATTR(false, true, 7);
#undef RTM_FOLD_ATTR
  cudaFuncSetAttribute(k_fold<true, true, 8, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)fold_smem_bytes(8));
  cudaFuncSetAttribute(k_fold<true, true, 7, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)fold_smem_bytes(7));
#define RTM_FOLD_ATTR_ND(SP_, BL_, CF_) \
  cudaFuncSetAttribute(k_fold<true, SP_, BL_, CF_, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)fold_smem_bytes(BL_))
  RTM_FOLD_ATTR_ND(true, 8, true); RTM_FOLD_ATTR_ND(true, 8, false); RTM_FOLD_ATTR_ND(false, 8, false);
  RTM_FOLD_ATTR_ND(true, 7, true); RTM_FOLD_ATTR_ND(true, 7, false); RTM_FOLD_ATTR_ND(false, 7, false);
#undef RTM_FOLD_ATTR_ND
  cudaFuncSetAttribute(k_fold_seq<true, 7, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)(sizeof(FoldSeqSmem<7>) * kFoldWarps));
  cudaFuncSetAttribute(k_fold_seq<true, 8, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)(sizeof(FoldSeqSmem<8>) * kFoldWarps));
  cudaFuncSetAttribute(k_fold_seq<true, 7>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)(sizeof(FoldSeqSmem<7>) * kFoldWarps));
  cudaFuncSetAttribute(k_fold_seq<false, 7>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)(sizeof(FoldSeqSmem<7>) * kFoldWarps));
  cudaFuncSetAttribute(k_fold_seq<true, 8>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)(sizeof(FoldSeqSmem<8>) * kFoldWarps));
  cudaFuncSetAttribute(k_fold_seq<false, 8>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)(sizeof(FoldSeqSmem<8>) * kFoldWarps));
  cudaGetLastError();
}

void launch_pack(const Params &p, void *pack, cudaStream_t st) {
  const PackLayout L = pack_layout(p);
  unsigned char *d = static_cast<unsigned char *>(pack);
  cudaMemcpyAsync(d + L.win, p.win, (size_t)kWinFields * p.W * 8, cudaMemcpyDeviceToDevice, st);
  cudaMemcpyAsync(d + L.topk, p.topk, (size_t)p.W * p.k * 8, cudaMemcpyDeviceToDevice, st);
  cudaMemcpyAsync(d + L.topk_n, p.topk_n, (size_t)p.W * 4, cudaMemcpyDeviceToDevice, st);
  cudaMemcpyAsync(d + L.kd, p.kdelta, (size_t)p.W * p.nk * 2 * 4, cudaMemcpyDeviceToDevice, st);
  if (p.rank_mode == RTM_RANK_MEAN) {
    if (p.tkey) cudaMemcpyAsync(d + L.tkey, p.tkey, (size_t)p.W * p.k * 8, cudaMemcpyDeviceToDevice, st);
    else cudaMemsetAsync(d + L.tkey, 0, (size_t)p.W * p.k * 8, st);
  }
}

uint64_t tables_bytes(const Params &p) { return tables_layout(p).total; }

void launch_pack_tables(const Params &p, void *pack, cudaStream_t st) {
  const TablesLayout L = tables_layout(p);
  unsigned char *d = static_cast<unsigned char *>(pack);
  { k_pack_tables<<<p.nc / 256 + 1 < 1184 ? p.nc / 256 + 1 : 1184, 256, 0, st>>>(p, d); count_launch(); }
  cudaMemcpyAsync(d + L.bstat, p.bstat, (size_t)p.nb * sizeof(rtm_buffer_stat), cudaMemcpyDeviceToDevice, st);
  if (p.pack_nb > p.nb)
    cudaMemsetAsync(d + L.bstat + (size_t)p.nb * sizeof(rtm_buffer_stat), 0,
                    (size_t)(p.pack_nb - p.nb) * sizeof(rtm_buffer_stat), st);
  if (p.gid) {
    cudaMemcpyAsync(d + L.gids, p.gid, (size_t)p.nb * 4, cudaMemcpyDeviceToDevice, st);
    if (p.pack_nb > p.nb) cudaMemsetAsync(d + L.gids + (size_t)p.nb * 4, 0xFF, (size_t)(p.pack_nb - p.nb) * 4, st);
  }
  cudaMemcpyAsync(d + L.hung, p.hung, (size_t)p.W * p.ncw * 4, cudaMemcpyDeviceToDevice, st);
}

void launch_merge_tables(const Params &p, const void *gathered, uint32_t world, cudaStream_t st) {
  { k_merge_tables<<<256, 256, 0, st>>>(p, static_cast<const unsigned char *>(gathered), world,
                                        tables_layout(p).total); count_launch(); }
}

void launch_scatter_bstat(const Params &p, cudaStream_t st) {
  const unsigned blocks = (p.nb + 255) / 256;
  { k_scatter_bstat<<<blocks < 1184 ? blocks : 1184, 256, 0, st>>>(p); count_launch(); }
}

// k_merge_windows holds next_pow2(world * k) candidates of 20 B in shared memory (opt-in 227 KB)
bool merge_fits(uint32_t world, uint32_t k) {
  uint64_t P = 1;
  while (P < (uint64_t)world * k) P <<= 1;
  return P * 20 <= 227ull * 1024;
}

void launch_merge(const Params &p, const void *gathered, uint32_t world, long long *gcum, cudaStream_t st) {
  const size_t stride = pack_layout(p).total;
  unsigned P = 1;
  while (P < world * p.k) P <<= 1;
  const size_t sm = (size_t)P * 20;  // cand + full_ent (u64) + sec (u32)
  if (sm > 48 * 1024) cudaFuncSetAttribute(k_merge_windows, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
  { k_merge_windows<<<p.W, 256, sm, st>>>(p, static_cast<const unsigned char *>(gathered), world, stride); count_launch(); }
  { k_merge_progress<<<p.nk, 1024, 0, st>>>(p, static_cast<const unsigned char *>(gathered), world, stride, gcum); count_launch(); }
}

#endif  // !RTM_TU_PARTITION
#ifdef RTM_TU_PARTITION  // the sample partition kernels' launchers: a module of their own
// (rtm_partition.cu); the partition kernels and their device helpers are compiled only there
template <int BL, bool CAPS, int KS, bool MP = false>
void launch_partition_lm(const Params &p, int n_sms, size_t sm, cudaStream_t st) {
  const int per_sm = occupancy((const void *)k_partition_lm<BL, CAPS, KS, MP>, kK1Threads, sm);
  unsigned grid = (unsigned)(n_sms * per_sm);
  const unsigned work = p.n_tiles_s + (p.fuse_events ? p.n_tiles_e : 0u);
  if (grid > work) grid = work;
  { k_partition_lm<BL, CAPS, KS, MP><<<grid, kK1Threads, sm, st>>>(p); count_launch(); }
}

void launch_partition(const Params &p, int n_sms, cudaStream_t st) {
  if (!p.n_tiles_s) return;
  if (p.nsb) {  // two-pass path, pass 1: superbin keys (capacities through L1: > 2^15 buffers)
    const bool caps = partition_caps_smem(p.nsb, p.nb);
    const size_t sm = k1_smem_lm(p.nsb, p.nb, caps);
    if (caps) launch_partition_lm<8, true, kSupLog>(p, n_sms, sm, st);
    else launch_partition_lm<8, false, kSupLog>(p, n_sms, sm, st);
    return;
  }
  const size_t sm = partition_smem_bytes(p.nbins, p.nb);
  if (p.nbins <= kLmMaxBins && p.bin_log == 7) {  // few-unit calls on a small registry
    if (partition_caps_smem(p.nbins, p.nb)) launch_partition_lm<8, true, 7>(p, n_sms, sm, st);
    else launch_partition_lm<8, false, 7>(p, n_sms, sm, st);
  } else if (p.nbins <= kLmMaxBins) {  // persistent: one or two CTAs per SM
    if (partition_caps_smem(p.nbins, p.nb)) launch_partition_lm<8, true, 8>(p, n_sms, sm, st);
    else launch_partition_lm<8, false, 8>(p, n_sms, sm, st);
  } else if (p.nbins < kTwoPassMinBins) {  // 171 .. 1023 bins: ranks in passes of <= 170 bins
    if (partition_caps_smem(p.nbins, p.nb)) launch_partition_lm<8, true, 8, true>(p, n_sms, sm, st);
    else launch_partition_lm<8, false, 8, true>(p, n_sms, sm, st);
  } else {
    if (p.bin_log == 7) { k_partition_mx<7><<<p.n_tiles_s, kK1Threads, sm, st>>>(p); count_launch(); }
    else { k_partition_mx<8><<<p.n_tiles_s, kK1Threads, sm, st>>>(p); count_launch(); }
  }
}

void configure_partition_once() {
  const int lm_caps = (int)k1_smem_lm(kLmMaxBins, 113 * 512, true);  // <= 113 KB by partition_caps_smem
  const int lm_glob = (int)k1_smem_lm(kLmMaxBins, 0, false);
  const int lm_mp = (int)k1_smem_lm(kTwoPassMinBins - 1, 0, false);
  cudaFuncSetAttribute(k_partition_lm<8, true, 8, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, lm_caps);
  cudaFuncSetAttribute(k_partition_lm<8, false, 8, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, lm_glob);
  cudaFuncSetAttribute(k_partition_lm<8, true, 7, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, lm_caps);
  cudaFuncSetAttribute(k_partition_lm<8, false, 7, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, lm_glob);
  cudaFuncSetAttribute(k_partition_lm<8, true, 8, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, lm_caps);
  cudaFuncSetAttribute(k_partition_lm<8, false, 8, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, lm_mp);
  cudaFuncSetAttribute(k_partition_lm<8, true, kSupLog, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, lm_caps);
  cudaFuncSetAttribute(k_partition_lm<8, false, kSupLog, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, lm_glob);
  cudaFuncSetAttribute(k_partition_mx<7>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)k1_smem_mx(kMaxBins));
  cudaFuncSetAttribute(k_partition_mx<8>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)k1_smem_mx(kMaxBins));
}
#endif  // RTM_TU_PARTITION
}  // namespace rtm
