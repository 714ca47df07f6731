// tools/microbench.cu — per-SM throughput of the warp primitives the partition scan uses.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/mb tools/microbench.cu && /tmp/mb
#include <cstdio>
#include <cuda_runtime.h>

constexpr int ITERS = 4096;

__global__ void k_match(unsigned *out, unsigned seed) {
  unsigned x = seed ^ threadIdx.x, acc = 0;
#pragma unroll 8
  for (int i = 0; i < ITERS; ++i) {
    unsigned key = (x >> 3) & 127u;
    unsigned m = __match_any_sync(0xFFFFFFFFu, key);
    acc += m;
    x = x * 1664525u + 1013904223u;  // independent of m: throughput, not latency
  }
  out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
}
__global__ void k_match_dep(unsigned *out, unsigned seed) {
  unsigned x = seed ^ threadIdx.x;
#pragma unroll 8
  for (int i = 0; i < ITERS; ++i) {
    unsigned m = __match_any_sync(0xFFFFFFFFu, x & 127u);
    x = (x * 1664525u + m) ^ (x >> 7);  // dependent chain: latency
  }
  out[blockIdx.x * blockDim.x + threadIdx.x] = x;
}
__global__ void k_ballot(unsigned *out, unsigned seed) {
  unsigned x = seed ^ threadIdx.x, acc = 0;
#pragma unroll 8
  for (int i = 0; i < ITERS; ++i) {
    acc += __ballot_sync(0xFFFFFFFFu, x & 8u);
    x = x * 1664525u + 1013904223u;
  }
  out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
}
__global__ void k_shfl(unsigned *out, unsigned seed) {
  unsigned x = seed ^ threadIdx.x, acc = 0;
#pragma unroll 8
  for (int i = 0; i < ITERS; ++i) {
    acc += __shfl_sync(0xFFFFFFFFu, x, (x >> 5) & 31);
    x = x * 1664525u + 1013904223u;
  }
  out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
}
__global__ void k_sts8(unsigned *out, unsigned seed) {
  __shared__ unsigned char buf[8192];
  unsigned x = seed ^ threadIdx.x;
#pragma unroll 8
  for (int i = 0; i < ITERS; ++i) {
    buf[(x >> 7) & 8191] = (unsigned char)x;
    x = x * 1664525u + 1013904223u;
  }
  __syncthreads();
  out[blockIdx.x * blockDim.x + threadIdx.x] = buf[threadIdx.x];
}
__global__ void k_popc_alu(unsigned *out, unsigned seed) {
  unsigned x = seed ^ threadIdx.x, acc = 0;
#pragma unroll 8
  for (int i = 0; i < ITERS; ++i) {
    acc += __popc(x & 0x5555u) + (x >> 3);
    x = x * 1664525u + 1013904223u;
  }
  out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
}

// MATCH restricted to a few lanes holding few distinct keys (the fold's duplicate lanes)
template <int ACTIVE_EVERY, int NKEYS>
__global__ void k_match_sparse(unsigned *out, unsigned seed) {
  unsigned x = seed ^ threadIdx.x, acc = 0;
  const unsigned lane = threadIdx.x & 31;
  const unsigned mask = __ballot_sync(0xFFFFFFFFu, lane % ACTIVE_EVERY == 0);
  if (lane % ACTIVE_EVERY == 0) {
#pragma unroll 8
    for (int i = 0; i < ITERS; ++i) {
      unsigned key = (x >> 3) % NKEYS;
      acc += __match_any_sync(mask, key);
      x = x * 1664525u + 1013904223u;
    }
  }
  out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
}

template <int BITS>
__device__ __forceinline__ unsigned match_ballot(unsigned key) {
  unsigned m = 0xFFFFFFFFu;
#pragma unroll
  for (int k = 0; k < BITS; ++k) {
    const unsigned b = __ballot_sync(0xFFFFFFFFu, (key >> k) & 1u);
    const unsigned s = 0u - ((key >> k) & 1u);  // all-ones when my bit is set
    m &= ~(b ^ s);
  }
  return m;
}
__global__ void k_match_ballot7(unsigned *out, unsigned seed) {
  unsigned x = seed ^ threadIdx.x, acc = 0;
#pragma unroll 8
  for (int i = 0; i < ITERS; ++i) {
    acc += match_ballot<7>((x >> 3) & 127u);
    x = x * 1664525u + 1013904223u;
  }
  out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
}
__global__ void k_match_ballot9(unsigned *out, unsigned seed) {
  unsigned x = seed ^ threadIdx.x, acc = 0;
#pragma unroll 8
  for (int i = 0; i < ITERS; ++i) {
    acc += match_ballot<9>((x >> 3) & 511u);
    x = x * 1664525u + 1013904223u;
  }
  out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
}

template <typename K>
void run(const char *name, K kern, int warps_per_sm, int n_ops_per_iter) {
  int sms = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  int clk = 0;
  cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
  unsigned *out;
  cudaMalloc(&out, sizeof(unsigned) * sms * warps_per_sm * 32);
  const int threads = warps_per_sm * 32 > 1024 ? 1024 : warps_per_sm * 32;
  const int blocks = sms * (warps_per_sm * 32 / threads);
  kern<<<blocks, threads>>>(out, 1);
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  cudaEventRecord(a);
  for (int r = 0; r < 5; ++r) kern<<<blocks, threads>>>(out, r);
  cudaEventRecord(b);
  cudaEventSynchronize(b);
  float ms = 0;
  cudaEventElapsedTime(&ms, a, b);
  const double warp_ops = 5.0 * blocks * (threads / 32) * ITERS * n_ops_per_iter;
  const double cycles = ms * 1e-3 * clk * 1e3;  // clock in kHz
  printf("%-12s warps/SM=%3d  %8.3f ms  %.2f warp-ops/cycle/SM  (%.1f cycles per warp-op per SM)\n", name,
         warps_per_sm, ms, warp_ops / cycles / sms, cycles * sms / warp_ops);
  cudaFree(out);
}

int main() {
  for (int w : {16, 32}) {
    run("match_ball7", k_match_ballot7, w, 1);
    run("match_ball9", k_match_ballot9, w, 1);
    run("match_any", k_match, w, 1);
    run("match_dep", k_match_dep, w, 1);
    run("m_all_2k", k_match_sparse<1, 2>, w, 1);
    run("m_all_8k", k_match_sparse<1, 8>, w, 1);
    run("m_8lane_2k", k_match_sparse<4, 2>, w, 1);
    run("m_4lane_2k", k_match_sparse<8, 2>, w, 1);
    run("m_4lane_4k", k_match_sparse<8, 4>, w, 1);
    run("ballot", k_ballot, w, 1);
    run("shfl_idx", k_shfl, w, 1);
    run("sts_u8", k_sts8, w, 1);
    run("alu_ref", k_popc_alu, w, 1);
  }
  return 0;
}
