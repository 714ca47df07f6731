/*
 * gen/rtm_gen.h — seeded, stateless, counter-based synthetic trace generator.
 *
 * This is INPUT infrastructure shared by the tests, the oracle harness and bench.py.
 * It holds none of the method's arithmetic (no folding, ranking, counting or hang
 * logic): it only says which record sits at stream index i.  Record i depends on
 * (params, i) alone, so host (gcc, gen_host.c) and device (nvcc, gen_cuda.cu)
 * produce bit-identical traces and shards can be regenerated instead of stored.
 *
 * Workload shape:
 *   - buffers are owned by components, owner(b) = b / buffers_per_comp
 *     (MGPUSim-like: every component has a few port buffers, Fig. 3);
 *   - capacities {4:35%, 8:35%, 16:15%, 128:10%, 1024:5%} mirror the paper's 4/8 port
 *     buffers (Fig. 3), 16-entry MSHR (L209), ~128-entry ROB (L205) and ~1000 RDMA (L211);
 *   - level classes: 90% normal, 5% fluctuating-high, 5% bottleneck (constantly full
 *     with rare dips, case study 1, L197-L199);
 *   - task events keep about `lag` tasks in flight; kernel = task / tasks_per_kernel
 *     (progress bars count thread blocks per kernel, L91, L131);
 *   - optional corruption (invalid_ppm) exercises drop counting.
 * ts is non-decreasing in the index: ts_i = t0 + floor(i * mul / 2^32).
 */
#ifndef RTM_GEN_H
#define RTM_GEN_H

#include <stdint.h>

#if defined(__CUDACC__)
#define GEN_HD __host__ __device__ __forceinline__
#else
#define GEN_HD static inline
#endif

typedef struct {
  int64_t ts;
  uint32_t buffer_id;
  uint16_t level;
  uint16_t capacity;
} gen_sample_rec; /* 16 B, same layout as rtm_level_sample */

typedef struct {
  int64_t ts;
  uint32_t task_id;
  uint32_t meta; /* component (bits 0..19) | kernel (bits 20..30) | kind (bit 31: 0 START, 1 END) */
} gen_event_rec; /* 16 B, same layout as rtm_task_event */

typedef struct {
  uint64_t seed;
  uint64_t n_samples;
  uint64_t n_events;
  int64_t t0;
  uint64_t ts_mul_s;          /* sample i at t0 + ((i * ts_mul_s) >> 32)            */
  uint64_t ts_mul_e;          /* event  j at t0 + ((j * ts_mul_e) >> 32)            */
  uint32_t n_buffers;
  uint32_t n_components;
  uint32_t n_kernels;
  uint32_t buffers_per_comp;  /* owner(b) = min(b / buffers_per_comp, n_components-1) */
  uint32_t lag;               /* tasks in flight                                     */
  uint32_t tasks_per_kernel;  /* kernel(task) = min(task / tpk, n_kernels - 1)       */
  uint32_t invalid_ppm;       /* corrupted records per million (0 = clean trace)     */
  uint32_t shard_world;       /* >1: keep only records whose owner comp % world == rank */
  uint32_t shard_rank;
  uint32_t zipf_n;            /* >0: buffer ids drawn by Zipf rank (C4), see gen_buffer_id    */
  uint64_t zipf_cdf;          /* address of u64 thresholds[zipf_n] (host or device memory,
                                 matching the fill), increasing, last = UINT64_MAX             */
  uint32_t zipf_a;            /* id = (rank * zipf_a + zipf_b) mod n_buffers (zipf_a coprime) */
  uint32_t zipf_b;
  int64_t dl_fill_ts[2];      /* deadlock stage s (C3): from dl_fill_ts[s] on, every sample of a
                                 buffer owned by dl_comp[2s], dl_comp[2s+1] is at capacity       */
  int64_t dl_quiet_ts[2];     /* ... and from dl_quiet_ts[s] on, their task events are
                                 redirected to component dl_sink (the stuck tasks stay in flight) */
  uint32_t dl_comp[4];
  uint32_t dl_sink;
  uint32_t n_dl_stages;       /* 0: no injection */
} rtm_gen_params;

/* ---- counter-based RNG: splitmix64 (Steele, Lea, Flood 2014) ---------------------- */
GEN_HD uint64_t gen_fmix64(uint64_t z) {
  z ^= z >> 30;
  z *= 0xbf58476d1ce4e5b9ULL;
  z ^= z >> 27;
  z *= 0x94d049bb133111ebULL;
  z ^= z >> 31;
  return z;
}
GEN_HD uint64_t gen_splitmix64(uint64_t x) { return gen_fmix64(x + 0x9E3779B97F4A7C15ULL); }
GEN_HD uint64_t gen_u(const rtm_gen_params *p, uint32_t stream, uint64_t i) {
  return gen_splitmix64(p->seed ^ ((uint64_t)stream << 56) ^ i);
}
/* Lemire: uniform in [0, n) from the low 32 bits of u */
GEN_HD uint32_t gen_below(uint64_t u, uint32_t n) {
  return (uint32_t)(((uint64_t)(uint32_t)u * (uint64_t)n) >> 32);
}
/* (a * b) >> 32 over the full 128-bit product, low 64 bits kept */
GEN_HD uint64_t gen_mulshr32(uint64_t a, uint64_t b) {
#if defined(__CUDA_ARCH__)
  uint64_t hi = __umul64hi(a, b);
  uint64_t lo = a * b;
#else
  unsigned __int128 pr = (unsigned __int128)a * (unsigned __int128)b;
  uint64_t hi = (uint64_t)(pr >> 64);
  uint64_t lo = (uint64_t)pr;
#endif
  return (hi << 32) | (lo >> 32);
}

enum { GEN_S_BUF = 1, GEN_S_CAP = 2, GEN_S_CLASS = 3, GEN_S_L1 = 4, GEN_S_L2 = 5, GEN_S_BAD = 6,
       GEN_S_COMP = 7, GEN_S_EBAD = 8 };

GEN_HD uint16_t gen_capacity(const rtm_gen_params *p, uint32_t b) {
  uint32_t h = (uint32_t)(gen_u(p, GEN_S_CAP, b) % 100u);
  return h < 35 ? 4 : h < 70 ? 8 : h < 85 ? 16 : h < 95 ? 128 : 1024;
}
/* 0 normal, 1 fluctuating-high, 2 bottleneck */
GEN_HD uint32_t gen_class(const rtm_gen_params *p, uint32_t b) {
  uint32_t h = (uint32_t)(gen_u(p, GEN_S_CLASS, b) % 100u);
  return h < 90 ? 0u : h < 95 ? 1u : 2u;
}
GEN_HD uint32_t gen_owner(const rtm_gen_params *p, uint32_t b) {
  uint32_t c = b / p->buffers_per_comp;
  return c < p->n_components ? c : p->n_components - 1;
}
GEN_HD uint32_t gen_task_comp(const rtm_gen_params *p, uint64_t task) {
  return gen_below(gen_u(p, GEN_S_COMP, task), p->n_components);
}
GEN_HD uint32_t gen_task_kernel(const rtm_gen_params *p, uint64_t task) {
  uint64_t k = task / p->tasks_per_kernel;
  return k < p->n_kernels ? (uint32_t)k : p->n_kernels - 1;
}

/* Buffer of sample i: uniform (Lemire), or Zipf over ranks by inverse CDF (binary search for
   the first threshold above u), ranks scattered over ids by an affine bijection (C4 hot spots
   land in unrelated components). */
GEN_HD uint32_t gen_buffer_id(const rtm_gen_params *p, uint64_t i) {
  uint64_t u = gen_u(p, GEN_S_BUF, i);
  if (!p->zipf_n) return gen_below(u, p->n_buffers);
  const uint64_t *cdf = (const uint64_t *)(uintptr_t)p->zipf_cdf;
  uint32_t lo = 0, hi = p->zipf_n - 1u; /* answer in [lo, hi] */
  while (lo < hi) {
    uint32_t mid = lo + (hi - lo) / 2u;
    if (u < cdf[mid]) hi = mid;
    else lo = mid + 1u;
  }
  return (uint32_t)(((uint64_t)lo * p->zipf_a + p->zipf_b) % p->n_buffers);
}
/* deadlock stage (0-based) of component c, or -1 */
GEN_HD int gen_dl_stage(const rtm_gen_params *p, uint32_t c) {
  for (uint32_t s = 0; s < p->n_dl_stages && s < 2u; ++s)
    if (c == p->dl_comp[2u * s] || c == p->dl_comp[2u * s + 1u]) return (int)s;
  return -1;
}

/* Level sample at stream index i (clean or, with invalid_ppm, possibly corrupted). */
GEN_HD gen_sample_rec gen_sample(const rtm_gen_params *p, uint64_t i) {
  gen_sample_rec r;
  uint32_t b = gen_buffer_id(p, i);
  uint16_t cap = gen_capacity(p, b);
  uint32_t cls = gen_class(p, b);
  uint64_t u1 = gen_u(p, GEN_S_L1, i), u2 = gen_u(p, GEN_S_L2, i);
  uint32_t lvl;
  if (cls == 0) {
    uint64_t m = u1 < u2 ? u1 : u2;
    lvl = (uint32_t)(m % (uint64_t)(cap + 1u));
  } else if (cls == 1) {
    lvl = cap - (uint32_t)(u1 % (uint64_t)(cap / 2u + 1u));
  } else {
    lvl = (u1 % 10u) != 0u ? cap : cap - 1u;
  }
  r.ts = p->t0 + (int64_t)gen_mulshr32(i, p->ts_mul_s);
  if (p->n_dl_stages) { /* injected circular wait: the stage's buffers back up and stay full */
    int s = gen_dl_stage(p, gen_owner(p, b));
    if (s >= 0 && r.ts >= p->dl_fill_ts[s]) lvl = cap;
  }
  r.buffer_id = b;
  r.level = (uint16_t)lvl;
  r.capacity = cap;
  if (p->invalid_ppm) {
    uint64_t u3 = gen_u(p, GEN_S_BAD, i);
    if ((uint32_t)(u3 % 1000000u) < p->invalid_ppm) {
      uint32_t kind = (uint32_t)((u3 >> 32) % 3u);
      if (kind == 0) r.buffer_id = p->n_buffers + (uint32_t)((u3 >> 40) % 1000u); /* unknown id */
      else if (kind == 1) r.level = (uint16_t)(cap + 1u + (uint32_t)((u3 >> 40) % 3u)); /* level > cap */
      else r.capacity = (uint16_t)(cap * 2u); /* capacity differs from the registered one */
    }
  }
  return r;
}

/* Task event at stream index j: first `lag` STARTs, then END(m/2) / START(lag + m/2) alternate. */
GEN_HD gen_event_rec gen_event(const rtm_gen_params *p, uint64_t j) {
  gen_event_rec r;
  uint64_t task;
  uint32_t kind;
  if (j < p->lag) {
    task = j;
    kind = 0;
  } else {
    uint64_t m = j - p->lag;
    if ((m & 1u) == 0) { task = m / 2; kind = 1; }
    else { task = p->lag + m / 2; kind = 0; }
  }
  uint32_t comp = gen_task_comp(p, task);
  uint32_t kern = gen_task_kernel(p, task);
  if (p->invalid_ppm) {
    uint64_t u3 = gen_u(p, GEN_S_EBAD, j);
    if ((uint32_t)(u3 % 1000000u) < p->invalid_ppm) {
      if ((u3 >> 32) & 1u) comp = p->n_components + (uint32_t)((u3 >> 40) % 7u);
      else if (p->n_kernels < 2048u) kern = p->n_kernels + (uint32_t)((u3 >> 40) % (2048u - p->n_kernels));
      else comp = p->n_components + 1u;
    }
  }
  r.ts = p->t0 + (int64_t)gen_mulshr32(j, p->ts_mul_e);
  if (p->n_dl_stages) { /* a deadlocked component neither starts nor finishes tasks */
    int s = gen_dl_stage(p, comp);
    if (s >= 0 && r.ts >= p->dl_quiet_ts[s]) comp = p->dl_sink;
  }
  r.task_id = (uint32_t)task;
  r.meta = (comp & 0xFFFFFu) | ((kern & 0x7FFu) << 20) | (kind << 31);
  if (comp > 0xFFFFFu) r.meta = 0xFFFFFu | ((kern & 0x7FFu) << 20) | (kind << 31);
  return r;
}

/* Sharding by owner component: record belongs to rank owner % world. */
GEN_HD int gen_sample_in_shard(const rtm_gen_params *p, const gen_sample_rec *r) {
  if (p->shard_world <= 1) return 1;
  uint32_t b = r->buffer_id < p->n_buffers ? r->buffer_id : 0u;
  return (gen_owner(p, b) % p->shard_world) == p->shard_rank;
}
GEN_HD int gen_event_in_shard(const rtm_gen_params *p, const gen_event_rec *r) {
  if (p->shard_world <= 1) return 1;
  uint32_t c = r->meta & 0xFFFFFu;
  if (c >= p->n_components) c = 0;
  return (c % p->shard_world) == p->shard_rank;
}

#endif /* RTM_GEN_H */
