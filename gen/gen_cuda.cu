// gen/gen_cuda.cu — device build of the synthetic trace generator (gen/rtm_gen.h).
// Input infrastructure for bench.py and the large-size parity tests: it writes a seeded
// trace straight into HBM (untimed).  No part of the monitored method lives here.
#include <cuda_runtime.h>
#include "rtm_gen.h"

namespace {

__global__ void gen_samples_kernel(rtm_gen_params p, uint64_t start, uint64_t count, gen_sample_rec *out) {
  uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t t = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; t < count; t += stride)
    out[t] = gen_sample(&p, start + t);
}

__global__ void gen_events_kernel(rtm_gen_params p, uint64_t start, uint64_t count, gen_event_rec *out) {
  uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t t = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; t < count; t += stride)
    out[t] = gen_event(&p, start + t);
}

// Shard filter: flag[t] = record in shard (compaction is done by the caller with a scan).
__global__ void gen_samples_flag_kernel(rtm_gen_params p, uint64_t start, uint64_t count, uint8_t *flag) {
  uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t t = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; t < count; t += stride) {
    gen_sample_rec r = gen_sample(&p, start + t);
    flag[t] = (uint8_t)gen_sample_in_shard(&p, &r);
  }
}

// Weak-scaling shards (bench.py, N > 1): rank r's local trace is mapped into the global id space
// of an N-times larger system, component-major: global comp = local comp * world + rank.
__global__ void remap_weak_kernel(gen_sample_rec *s, uint64_t ns, gen_event_rec *e, uint64_t ne, uint32_t nbl,
                                  uint32_t ncl, uint32_t bpc, uint32_t rank, uint32_t world) {
  uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t t = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; t < ns; t += stride) {
    uint32_t b = s[t].buffer_id;
    if (b < nbl) {
      uint32_t gc = (b / bpc) * world + rank;
      s[t].buffer_id = gc * bpc + b % bpc;
    } else {
      s[t].buffer_id = 0xFFFFFFF0u;
    }
  }
  for (uint64_t t = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; t < ne; t += stride) {
    uint32_t m = e[t].meta, c = m & 0xFFFFFu;
    uint32_t gc = c < ncl ? c * world + rank : 0xFFFFFu;
    e[t].meta = (m & ~0xFFFFFu) | (gc & 0xFFFFFu);
  }
}

int grid_for(uint64_t count) {
  uint64_t g = (count + 255) / 256;
  return (int)(g > 148 * 32 ? 148 * 32 : (g ? g : 1));
}

}  // namespace

extern "C" {

// Unfiltered device fill (shard_world is ignored); returns a cudaError_t.
int gen_cuda_fill_samples(const rtm_gen_params *p, uint64_t start, uint64_t count, void *out, void *stream) {
  if (count == 0) return 0;
  gen_samples_kernel<<<grid_for(count), 256, 0, (cudaStream_t)stream>>>(*p, start, count, (gen_sample_rec *)out);
  return (int)cudaGetLastError();
}

int gen_cuda_fill_events(const rtm_gen_params *p, uint64_t start, uint64_t count, void *out, void *stream) {
  if (count == 0) return 0;
  gen_events_kernel<<<grid_for(count), 256, 0, (cudaStream_t)stream>>>(*p, start, count, (gen_event_rec *)out);
  return (int)cudaGetLastError();
}

int gen_cuda_flag_samples(const rtm_gen_params *p, uint64_t start, uint64_t count, void *flag, void *stream) {
  if (count == 0) return 0;
  gen_samples_flag_kernel<<<grid_for(count), 256, 0, (cudaStream_t)stream>>>(*p, start, count, (uint8_t *)flag);
  return (int)cudaGetLastError();
}

int gen_cuda_remap_weak(const rtm_gen_params *p, void *s, uint64_t ns, void *e, uint64_t ne, uint32_t rank,
                        uint32_t world, void *stream) {
  uint64_t m = ns > ne ? ns : ne;
  remap_weak_kernel<<<grid_for(m), 256, 0, (cudaStream_t)stream>>>((gen_sample_rec *)s, ns, (gen_event_rec *)e, ne,
                                                                   p->n_buffers, p->n_components,
                                                                   p->buffers_per_comp, rank, world);
  return (int)cudaGetLastError();
}

// Copy a host table (e.g. the Zipf thresholds) into a new device allocation (kept for the process).
int gen_cuda_upload(const void *host, uint64_t bytes, void **out) {
  void *d = nullptr;
  cudaError_t e = cudaMalloc(&d, bytes ? bytes : 1);
  if (e != cudaSuccess) return (int)e;
  e = cudaMemcpy(d, host, bytes, cudaMemcpyHostToDevice);
  if (e != cudaSuccess) return (int)e;
  *out = d;
  return 0;
}

}  // extern "C"
