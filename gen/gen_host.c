/*
 * gen/gen_host.c — host (gcc) build of the synthetic trace generator (gen/rtm_gen.h).
 * Input infrastructure only: no part of the monitored method lives here.
 */
#include "rtm_gen.h"

/* Writes the records of indices [start, start+count) that belong to the shard; returns how many. */
uint64_t gen_fill_samples(const rtm_gen_params *p, uint64_t start, uint64_t count, gen_sample_rec *out) {
  uint64_t n = 0;
  for (uint64_t i = start; i < start + count; ++i) {
    gen_sample_rec r = gen_sample(p, i);
    if (gen_sample_in_shard(p, &r)) out[n++] = r;
  }
  return n;
}

uint64_t gen_fill_events(const rtm_gen_params *p, uint64_t start, uint64_t count, gen_event_rec *out) {
  uint64_t n = 0;
  for (uint64_t j = start; j < start + count; ++j) {
    gen_event_rec r = gen_event(p, j);
    if (gen_event_in_shard(p, &r)) out[n++] = r;
  }
  return n;
}

/* Registry that a simulator would register at start-up (RegisterComponent / CreateProgressBar). */
void gen_fill_registry(const rtm_gen_params *p, uint32_t *owner, uint16_t *capacity, int64_t *kernel_total) {
  for (uint32_t b = 0; b < p->n_buffers; ++b) {
    if (owner) owner[b] = gen_owner(p, b);
    if (capacity) capacity[b] = gen_capacity(p, b);
  }
  if (kernel_total)
    for (uint32_t k = 0; k < p->n_kernels; ++k) kernel_total[k] = (int64_t)p->tasks_per_kernel;
}

uint64_t gen_splitmix64_c(uint64_t x) { return gen_splitmix64(x); }
