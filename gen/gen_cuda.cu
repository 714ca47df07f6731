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

}  // extern "C"
