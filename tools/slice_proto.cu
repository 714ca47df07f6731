// Prototype / microbenchmark: sliced window-range fold (no partition pass).
// CTA (range r, slice s) scans every sample record of its window range, compacts the ones whose
// buffer lies in its slice, and folds them in ingest order against per-buffer state in shared
// memory (duplicates inside a tile take a warp-serial path).  Measures throughput only.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -o tools/slice_proto tools/slice_proto.cu
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <vector>

#define CK(x) do { cudaError_t e_ = (x); if (e_ != cudaSuccess) { printf("CUDA %s at %d\n", cudaGetErrorString(e_), __LINE__); exit(1); } } while (0)

constexpr int TPB = 512;
constexpr int TILE = 1024;  // records per tile (2 per thread)
constexpr unsigned kFull = 0xFFFFFFFFu;

struct P {
  const int4 *rec;
  const long long *B;   // [W+1] record boundaries
  const long long *T;   // [W+1] tick boundaries
  const uint16_t *cap;
  const uint32_t *owner;
  uint32_t nb, W, R, SL;
  uint16_t *lastlvl;
  uint32_t *anyfull;
  uint32_t ncw;
  unsigned long long *dig;
  uint4 *pend;
};

__device__ __forceinline__ unsigned lanemask_lt() { unsigned m; asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m)); return m; }

template <int S>
__global__ void __launch_bounds__(TPB, 2) k_slice(P p) {
  extern __shared__ __align__(16) unsigned char sm[];
  const unsigned SL = p.SL;
  uint4 *st = (uint4 *)sm;                               // [SL]  I lo, I hi, L|mx<<16, mn|n<<16
  uint2 *comp = (uint2 *)(st + SL);                      // [TILE] off32, lb | lvl<<16 (lb<2^14)... idx in dupidx
  uint16_t *cidx = (uint16_t *)(comp + TILE);            // [TILE] tile index of comp entry
  uint16_t *capS = cidx + TILE;                          // [SL]
  uint32_t *bm = (uint32_t *)(capS + ((SL + 7) & ~7u));  // seen[2][SL/32], dupb[2][SL/32]
  const unsigned nw = SL / 32;
  uint32_t *dupmask = bm + 4 * nw;                       // [TILE/32] dup entries by tile index
  uint16_t *dupj = (uint16_t *)(dupmask + TILE / 32);    // [TILE] comp position of the dup at idx
  __shared__ unsigned s_cnt, s_ndup;

  const unsigned r = blockIdx.x / S, s = blockIdx.x % S;
  const unsigned base = s * SL;
  const unsigned w0 = (unsigned)((unsigned long long)r * p.W / p.R), w1 = (unsigned)((unsigned long long)(r + 1) * p.W / p.R);
  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  for (unsigned i = tid; i < SL; i += TPB) {
    st[i] = make_uint4(0, 0, 0, 0);
    capS[i] = base + i < p.nb ? p.cap[base + i] : 1;
  }
  for (unsigned i = tid; i < 4 * nw + TILE / 32; i += TPB) bm[i] = 0;
  if (tid == 0) s_cnt = 0;
  __syncthreads();
  unsigned tseq = 0;
  for (unsigned w = w0; w < w1; ++w) {
    const long long a = p.B[w], b = p.B[w + 1];
    const long long te = p.T[w + 1];
    const unsigned long long Wlen = (unsigned long long)(te - p.T[w]);
    // window init: I = L * Wlen, mx = mn = L, n = 0  (done at previous finalize; first window: L=0)
    int4 r0, r1;
    long long pos = a;
    auto ld = [&](long long q) -> int4 { return q < b ? __ldcs(p.rec + q) : make_int4(0, 0, -1, 0); };
    r0 = ld(pos + tid);
    r1 = ld(pos + tid + TPB);
    for (; pos < b; pos += TILE, ++tseq) {
      const int4 n0 = ld(pos + TILE + tid), n1 = ld(pos + TILE + TPB + tid);
      // ---- phase A: compact in-slice records (ballot), validity from the slice's cap table
      const unsigned set = tseq & 1;
      uint32_t *seen = bm + set * nw, *dupb = bm + (2 + set) * nw;
#pragma unroll
      for (int q = 0; q < 2; ++q) {
        const int4 v = q ? r1 : r0;
        const unsigned lb = (unsigned)v.z - base;
        bool in = lb < SL;
        if (in) {
          const unsigned lvl = (unsigned)v.w & 0xFFFFu, c = (unsigned)v.w >> 16;
          in = (c == capS[lb]) & (lvl <= c);
        }
        const unsigned m = __ballot_sync(kFull, in);
        unsigned basepos = 0;
        if (lane == 0 && m) basepos = atomicAdd(&s_cnt, __popc(m));
        basepos = __shfl_sync(kFull, basepos, 0);
        if (in) {
          const unsigned j = basepos + __popc(m & lanemask_lt());
          const long long ts = ((long long)(unsigned)v.y << 32) | (unsigned)v.x;
          comp[j] = make_uint2((unsigned)(te - ts), lb | (((unsigned)v.w & 0xFFFFu) << 16));
          cidx[j] = (uint16_t)(q * TPB + tid);
        }
      }
      __syncthreads();
      const unsigned cnt = s_cnt;
      // ---- phase B: duplicate detection (bitmaps)
      for (unsigned j = tid; j < cnt; j += TPB) {
        const unsigned lb = comp[j].y & 0xFFFFu, m = 1u << (lb & 31);
        const unsigned old = atomicOr(seen + (lb >> 5), m);
        if (old & m) atomicOr(dupb + (lb >> 5), m);
      }
      __syncthreads();
      // ---- phase C: singles update state; dups registered by tile index
      if (tid == 0) s_cnt = 0;
      for (unsigned j = tid; j < cnt; j += TPB) {
        const uint2 e = comp[j];
        const unsigned lb = e.y & 0xFFFFu, lvl = e.y >> 16, m = 1u << (lb & 31);
        if (dupb[lb >> 5] & m) {
          const unsigned x = cidx[j];
          dupj[x] = (uint16_t)j;
          atomicOr(dupmask + (x >> 5), 1u << (x & 31));
        } else {
          uint4 sv = st[lb];
          const unsigned L = sv.z & 0xFFFFu;
          unsigned long long I = ((unsigned long long)sv.y << 32) | sv.x;
          I += (unsigned long long)((long long)((int)lvl - (int)L) * (long long)e.x);
          const unsigned mx = max(sv.z >> 16, lvl), mn = min(sv.w & 0xFFFFu, lvl);
          st[lb] = make_uint4((unsigned)I, (unsigned)(I >> 32), lvl | (mx << 16), mn | ((sv.w & 0xFFFF0000u) + 0x10000u));
        }
      }
      // clear the other bitmap set for the next tile
      for (unsigned i = tid; i < 2 * nw; i += TPB) bm[(i < nw ? (set ^ 1) * nw : (2 + (set ^ 1)) * nw - nw) + i] = 0;
      __syncthreads();
      // ---- dups: warp 0, in tile-index order
      if (wid == 0) {
        for (int wd = 0; wd < TILE / 32; ++wd) {
          const unsigned dm = dupmask[wd];
          if (!dm) continue;
          const bool act = (dm >> lane) & 1u;
          unsigned lb = 0xFFFFFFFFu, lvl = 0, off = 0;
          if (act) {
            const uint2 e = comp[dupj[wd * 32 + lane]];
            lb = e.y & 0xFFFFu;
            lvl = e.y >> 16;
            off = e.x;
          }
          const unsigned peers = __match_any_sync(kFull, lb);
          const unsigned rank = __popc(peers & lanemask_lt());
          const unsigned maxr = __reduce_max_sync(kFull, act ? rank : 0u);
          for (unsigned k = 0; k <= maxr; ++k) {
            if (act && rank == k) {
              uint4 sv = st[lb];
              const unsigned L = sv.z & 0xFFFFu;
              unsigned long long I = ((unsigned long long)sv.y << 32) | sv.x;
              I += (unsigned long long)((long long)((int)lvl - (int)L) * (long long)off);
              const unsigned mx = max(sv.z >> 16, lvl), mn = min(sv.w & 0xFFFFu, lvl);
              st[lb] = make_uint4((unsigned)I, (unsigned)(I >> 32), lvl | (mx << 16), mn | ((sv.w & 0xFFFF0000u) + 0x10000u));
            }
            __syncwarp();
          }
          if (lane == 0) dupmask[wd] = 0;
        }
      }
      // (the next tile's phase A writes comp: warp 0 must be done -> barrier)
      __syncthreads();
      r0 = n0;
      r1 = n1;
    }
    // ---- finalize the window for the slice
    const unsigned long long Wn = w + 1 < p.W ? (unsigned long long)(p.T[w + 2] - te) : 0ull;
    unsigned long long dig = 0;
    for (unsigned i = tid; i < SL; i += TPB) {
      const unsigned bb = base + i;
      if (bb >= p.nb) break;
      const uint4 sv = st[i];
      const unsigned L = sv.z & 0xFFFFu, mx = sv.z >> 16, mn = sv.w & 0xFFFFu, n = sv.w >> 16;
      const unsigned long long I = ((unsigned long long)sv.y << 32) | sv.x;
      p.lastlvl[(size_t)w * p.nb + bb] = (uint16_t)L;
      if (mn == capS[i]) {
        const unsigned c = __ldg(p.owner + bb);
        atomicOr(p.anyfull + (size_t)w * p.ncw + (c >> 5), 1u << (c & 31));
      }
      if (n) {
        unsigned long long h = (I * 0x9E3779B97F4A7C15ULL) ^ ((((unsigned long long)n << 32) | bb) * 0xC2B2AE3D27D4EB4FULL) ^
                               (((unsigned long long)L | ((unsigned long long)mx << 16) | ((unsigned long long)mn << 32) |
                                 ((unsigned long long)capS[i] << 48)) * 0x165667B19E3779F9ULL);
        h ^= h >> 30; h *= 0xbf58476d1ce4e5b9ULL; h ^= h >> 27; h *= 0x94d049bb133111ebULL; h ^= h >> 31;
        dig += h;
      }
      const unsigned long long In = (unsigned long long)L * Wn;
      st[i] = make_uint4((unsigned)In, (unsigned)(In >> 32), L | (L << 16), L);
    }
    for (int o = 16; o; o >>= 1) dig += __shfl_xor_sync(kFull, dig, o);
    if (lane == 0 && dig) atomicAdd(p.dig + w, dig);
    __syncthreads();
  }
}

static unsigned long long sm64(unsigned long long x) {
  x += 0x9E3779B97F4A7C15ULL; x = (x ^ (x >> 30)) * 0xbf58476d1ce4e5b9ULL; x = (x ^ (x >> 27)) * 0x94d049bb133111ebULL; return x ^ (x >> 31);
}

template <int S>
float run(P p, int n_sms) {
  p.SL = ((p.nb + S - 1) / S + 31) & ~31u;
  const unsigned nw = p.SL / 32;
  size_t smem = (size_t)p.SL * 16 + TILE * 8 + TILE * 2 + ((p.SL + 7) & ~7u) * 2 + (4 * nw + TILE / 32) * 4 + TILE * 2 + 64;
  if (smem > 227 * 1024) { printf("S=%d: smem %zu too large\n", S, smem); return 0; }
  CK(cudaFuncSetAttribute(k_slice<S>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  int occ = 0;
  CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_slice<S>, TPB, smem));
  p.R = (n_sms * occ) / S;
  if (p.R > p.W) p.R = p.W;
  cudaEvent_t e0, e1;
  CK(cudaEventCreate(&e0)); CK(cudaEventCreate(&e1));
  float best = 1e9;
  for (int it = 0; it < 6; ++it) {
    CK(cudaEventRecord(e0));
    k_slice<S><<<p.R * S, TPB, smem>>>(p);
    CK(cudaEventRecord(e1));
    CK(cudaEventSynchronize(e1));
    float ms; CK(cudaEventElapsedTime(&ms, e0, e1));
    if (it) best = ms < best ? ms : best;
  }
  CK(cudaGetLastError());
  printf("S=%d SL=%u smem=%zu occ=%d R=%u : %.3f ms\n", S, p.SL, smem, occ, p.R, best);
  return best;
}

int main(int argc, char **argv) {
  const uint32_t nb = argc > 1 ? atoi(argv[1]) : 20480;
  const long long N = argc > 2 ? atoll(argv[2]) : 90000000LL;
  const uint32_t W = 1000;
  std::vector<uint16_t> cap(nb);
  std::vector<uint32_t> owner(nb);
  const uint16_t caps[5] = {4, 8, 16, 128, 1024};
  for (uint32_t b = 0; b < nb; ++b) { cap[b] = caps[sm64(b) % 5]; owner[b] = b / 4; }
  std::vector<int4> h(N);
  for (long long i = 0; i < N; ++i) {
    unsigned long long u = sm64(i * 7 + 1);
    unsigned b = (unsigned)((u & 0xFFFFFFFFull) * nb >> 32);
    unsigned c = cap[b], l = (unsigned)((u >> 32) % (c + 1));
    long long ts = i / 2;
    h[i] = make_int4((int)(unsigned)ts, (int)(ts >> 32), (int)b, (int)(l | (c << 16)));
  }
  std::vector<long long> B(W + 1), T(W + 1);
  for (uint32_t w = 0; w <= W; ++w) { T[w] = (long long)w * (N / 2) / W; B[w] = 2 * T[w]; }
  P p{};
  int4 *drec; CK(cudaMalloc(&drec, N * 16)); CK(cudaMemcpy(drec, h.data(), N * 16, cudaMemcpyHostToDevice));
  long long *dB, *dT; CK(cudaMalloc(&dB, (W + 1) * 8)); CK(cudaMalloc(&dT, (W + 1) * 8));
  CK(cudaMemcpy(dB, B.data(), (W + 1) * 8, cudaMemcpyHostToDevice)); CK(cudaMemcpy(dT, T.data(), (W + 1) * 8, cudaMemcpyHostToDevice));
  uint16_t *dcap; CK(cudaMalloc(&dcap, nb * 2)); CK(cudaMemcpy(dcap, cap.data(), nb * 2, cudaMemcpyHostToDevice));
  uint32_t *down; CK(cudaMalloc(&down, nb * 4)); CK(cudaMemcpy(down, owner.data(), nb * 4, cudaMemcpyHostToDevice));
  p.rec = drec; p.B = dB; p.T = dT; p.cap = dcap; p.owner = down; p.nb = nb; p.W = W;
  p.ncw = (nb / 4 + 31) / 32;
  CK(cudaMalloc(&p.lastlvl, (size_t)W * nb * 2));
  CK(cudaMalloc(&p.anyfull, (size_t)W * p.ncw * 4));
  CK(cudaMalloc(&p.dig, W * 8));
  int n_sms; CK(cudaDeviceGetAttribute(&n_sms, cudaDevAttrMultiProcessorCount, 0));
  printf("nb=%u N=%lld W=%u sms=%d  (HBM floor at 6.4 TB/s: %.3f ms)\n", nb, N, W, n_sms, N * 16 / 6.4e9);
  run<1>(p, n_sms);
  run<2>(p, n_sms);
  run<4>(p, n_sms);
  run<8>(p, n_sms);
  return 0;
}
