/*
 * oracle/oracle.c — plain single-threaded C oracle (TEST INFRASTRUCTURE ONLY; see oracle.h).
 *
 * Follows DESIGN.md §2 ("what a window snapshot is") step by step, window by window, with
 * no blocking, fusion or reordering: a sequential per-buffer fold in ingest order, a full
 * sort for the Bottleneck Analyzer list, plain counters for the progress bars and a
 * run-length counter per component for the hang flag.  Integer results are exact
 * (the integral is int64, wrapping mod 2^64 like the CUDA path); the one ratio, mean
 * occupancy, is a single IEEE division.
 */
#include "oracle.h"

#include <stdlib.h>
#include <string.h>

struct orc_ctx {
  uint32_t nb, nc, nk;
  uint32_t *owner;
  uint16_t *cap;
  int64_t *ktotal;
  uint8_t *owned;
  uint32_t H, k;
  int32_t rank_mode, hang_mode;
  int64_t t0, t_prev;
  uint16_t *lvl;       /* level of every buffer at the end of the last reduced window */
  int64_t *c_started, *c_ended, *k_started, *k_ended;
  uint32_t *run;       /* consecutive windows with cond_c true */
  uint32_t *persist;   /* per buffer: windows in which it was in the top-k list */
  uint8_t *live;       /* progress bar id in use (Create/DestroyProgressBar, L99) */
  int64_t *ktotal0;    /* bar totals as registered at create (restored by reset) */
  int sticky;
};

/* ---- digest mixer (DESIGN.md §2 "digest", reading R17): three fields folded by odd-constant
 * products (bijections of Z/2^64), XORed, then one splitmix64 finalizer.  A change in any single
 * field changes the term. ---- */
static uint64_t fmix64(uint64_t z) {
  z ^= z >> 30;
  z *= 0xbf58476d1ce4e5b9ULL;
  z ^= z >> 27;
  z *= 0x94d049bb133111ebULL;
  z ^= z >> 31;
  return z;
}

uint64_t orc_digest_term(uint32_t b, uint16_t last, uint16_t mx, uint16_t mn, uint16_t cap, uint32_t n,
                         int64_t integral) {
  const uint64_t levels = (uint64_t)last | ((uint64_t)mx << 16) | ((uint64_t)mn << 32) | ((uint64_t)cap << 48);
  const uint64_t ident = ((uint64_t)n << 32) | (uint64_t)b;
  return fmix64(((uint64_t)integral * 0x9E3779B97F4A7C15ULL) ^ (ident * 0xC2B2AE3D27D4EB4FULL) ^
                (levels * 0x165667B19E3779F9ULL));
}

orc_ctx *orc_create(const orc_config *cfg) {
  if (!cfg || cfg->n_buffers == 0 || cfg->n_components == 0 || cfg->n_kernels == 0 || cfg->n_kernels > 2048 ||
      cfg->n_components > (1u << 20) || cfg->n_buffers > 0x7FFFFFFFu || cfg->hang_windows == 0 ||
      !cfg->buffer_owner || !cfg->buffer_capacity || !cfg->kernel_total)
    return NULL;
  for (uint32_t b = 0; b < cfg->n_buffers; ++b)
    if (cfg->buffer_capacity[b] == 0 || cfg->buffer_owner[b] >= cfg->n_components) return NULL;
  orc_ctx *c = (orc_ctx *)calloc(1, sizeof(orc_ctx));
  c->nb = cfg->n_buffers;
  c->nc = cfg->n_components;
  c->nk = cfg->n_kernels;
  c->owner = (uint32_t *)malloc(sizeof(uint32_t) * c->nb);
  c->cap = (uint16_t *)malloc(sizeof(uint16_t) * c->nb);
  c->ktotal = (int64_t *)malloc(sizeof(int64_t) * c->nk);
  c->owned = (uint8_t *)malloc(c->nc);
  memcpy(c->owner, cfg->buffer_owner, sizeof(uint32_t) * c->nb);
  memcpy(c->cap, cfg->buffer_capacity, sizeof(uint16_t) * c->nb);
  memcpy(c->ktotal, cfg->kernel_total, sizeof(int64_t) * c->nk);
  for (uint32_t i = 0; i < c->nc; ++i) c->owned[i] = cfg->owned ? (cfg->owned[i] != 0) : 1;
  c->H = cfg->hang_windows;
  c->k = cfg->k;
  c->rank_mode = cfg->rank_mode;
  c->hang_mode = cfg->hang_mode;
  c->t0 = cfg->t0;
  c->lvl = (uint16_t *)malloc(sizeof(uint16_t) * c->nb);
  c->c_started = (int64_t *)malloc(sizeof(int64_t) * c->nc);
  c->c_ended = (int64_t *)malloc(sizeof(int64_t) * c->nc);
  c->k_started = (int64_t *)malloc(sizeof(int64_t) * c->nk);
  c->k_ended = (int64_t *)malloc(sizeof(int64_t) * c->nk);
  c->run = (uint32_t *)malloc(sizeof(uint32_t) * c->nc);
  c->persist = (uint32_t *)malloc(sizeof(uint32_t) * (c->nb ? c->nb : 1));
  c->live = (uint8_t *)malloc(c->nk ? c->nk : 1);
  c->ktotal0 = (int64_t *)malloc(sizeof(int64_t) * (c->nk ? c->nk : 1));
  memcpy(c->ktotal0, cfg->kernel_total, sizeof(int64_t) * c->nk);
  orc_reset(c);
  return c;
}

void orc_reset(orc_ctx *c) {
  c->t_prev = c->t0;
  memset(c->lvl, 0, sizeof(uint16_t) * c->nb); /* buffers start empty */
  memset(c->c_started, 0, sizeof(int64_t) * c->nc);
  memset(c->c_ended, 0, sizeof(int64_t) * c->nc);
  memset(c->k_started, 0, sizeof(int64_t) * c->nk);
  memset(c->k_ended, 0, sizeof(int64_t) * c->nk);
  memset(c->run, 0, sizeof(uint32_t) * c->nc);
  memset(c->persist, 0, sizeof(uint32_t) * c->nb);
  memset(c->live, 1, c->nk); /* every registered bar is live */
  memcpy(c->ktotal, c->ktotal0, sizeof(int64_t) * c->nk);
  c->sticky = 0;
}

void orc_destroy(orc_ctx *c) {
  if (!c) return;
  free(c->owner); free(c->cap); free(c->ktotal); free(c->owned); free(c->lvl);
  free(c->c_started); free(c->c_ended); free(c->k_started); free(c->k_ended); free(c->run); free(c->persist);
  free(c->live); free(c->ktotal0);
  free(c);
}

/* smallest w with ts < t_end[w]; caller guarantees t_begin <= ts < t_end[W-1] */
static uint32_t window_of(const int64_t *t_end, uint32_t W, int64_t ts) {
  uint32_t lo = 0, hi = W - 1;
  while (lo < hi) {
    uint32_t mid = lo + (hi - lo) / 2;
    if (ts < t_end[mid]) hi = mid; else lo = mid + 1;
  }
  return lo;
}

/* Bottleneck Analyzer order: fullness percentage (or element count),
 * descending; equal fullness -> buffer_id ascending.  Ratios compared exactly by
 * cross-multiplication: a.l/a.c > b.l/b.c  <=>  a.l*b.c > b.l*a.c. */
typedef struct { uint32_t id; uint16_t l, c; uint64_t I; } rank_item;
static int cmp_percent(const void *pa, const void *pb) {
  const rank_item *a = (const rank_item *)pa, *b = (const rank_item *)pb;
  uint64_t x = (uint64_t)a->l * b->c, y = (uint64_t)b->l * a->c;
  if (x != y) return x > y ? -1 : 1;
  return a->id < b->id ? -1 : (a->id > b->id ? 1 : 0);
}
/* Persistence ranking ("repeatedly at the top", L173, L197-L199): the
 * window's time-weighted mean occupancy I / (cap * W), descending; within one window W is
 * common, so I_a/c_a > I_b/c_b  <=>  I_a*c_b > I_b*c_a (128-bit products, exact). */
static int cmp_mean(const void *pa, const void *pb) {
  const rank_item *a = (const rank_item *)pa, *b = (const rank_item *)pb;
  unsigned __int128 x = (unsigned __int128)a->I * b->c, y = (unsigned __int128)b->I * a->c;
  if (x != y) return x > y ? -1 : 1;
  return a->id < b->id ? -1 : (a->id > b->id ? 1 : 0);
}
static int cmp_size(const void *pa, const void *pb) {
  const rank_item *a = (const rank_item *)pa, *b = (const rank_item *)pb;
  if (a->l != b->l) return a->l > b->l ? -1 : 1;
  return a->id < b->id ? -1 : (a->id > b->id ? 1 : 0);
}

/* Stream classification (DESIGN.md §2 "ingest"): kept window or drop, attribution of drops. */
static int classify(int is_sample, const void *recs, uint64_t n, const orc_ctx *c, const int64_t *t_end,
                    uint32_t W, int64_t t_begin, int32_t *win, uint64_t *dropped) {
  const orc_sample *s = (const orc_sample *)recs;
  const orc_event *e = (const orc_event *)recs;
  /* pass 1: field validity and the ts-order contract over field-valid records */
  int have_prev = 0;
  int64_t prev_ts = 0;
  for (uint64_t i = 0; i < n; ++i) {
    int valid;
    int64_t ts;
    if (is_sample) {
      valid = s[i].buffer_id < c->nb && s[i].capacity == c->cap[s[i].buffer_id] && s[i].level <= s[i].capacity;
      ts = s[i].ts;
    } else {
      uint32_t comp = e[i].meta & 0xFFFFFu, kern = (e[i].meta >> 20) & 0x7FFu;
      valid = comp < c->nc && kern < c->nk && c->live[kern]; /* a destroyed bar takes no events */
      ts = e[i].ts;
    }
    if (valid) {
      if (have_prev && ts < prev_ts) return -4;
      prev_ts = ts;
      have_prev = 1;
      if (ts < t_begin) win[i] = -1;              /* late: dropped, charged to window 0 */
      else if (ts >= t_end[W - 1]) win[i] = -2;   /* early: dropped, charged to window W-1 */
      else win[i] = (int32_t)window_of(t_end, W, ts);
    } else {
      win[i] = -3;                                /* field-invalid */
    }
  }
  /* pass 2 (backwards): a dropped record is charged to the window of the next field-valid
   * record in the stream (late -> 0, early -> W-1); trailing invalid records -> W-1. */
  uint32_t next_charge = W - 1;
  for (uint64_t r = n; r-- > 0;) {
    int32_t v = win[r];
    if (v >= 0) next_charge = (uint32_t)v;
    else if (v == -1) { next_charge = 0; dropped[0]++; }
    else if (v == -2) { next_charge = W - 1; dropped[W - 1]++; }
    else dropped[next_charge]++;
  }
  return 0;
}

/* stable bucketing of kept record indices by window */
static void bucket(const int32_t *win, uint64_t n, uint32_t W, uint64_t *start, uint64_t *order) {
  memset(start, 0, sizeof(uint64_t) * (W + 1));
  for (uint64_t i = 0; i < n; ++i) if (win[i] >= 0) start[win[i] + 1]++;
  for (uint32_t w = 0; w < W; ++w) start[w + 1] += start[w];
  uint64_t *fill = (uint64_t *)malloc(sizeof(uint64_t) * (W + 1));
  memcpy(fill, start, sizeof(uint64_t) * (W + 1));
  for (uint64_t i = 0; i < n; ++i) if (win[i] >= 0) order[fill[win[i]]++] = i;
  free(fill);
}

int orc_reduce(orc_ctx *c, const orc_sample *s, uint64_t ns, const orc_event *e, uint64_t ne,
               const int64_t *t_end, uint32_t W, orc_summary *sum, orc_topk *topk, uint32_t *topk_n,
               orc_progress *prog, uint8_t *hung, orc_bstat *last_stats, orc_comp *comps,
               orc_bstat *all_stats) {
  if (!c) return -1;
  if (c->sticky) return c->sticky;
  if (W == 0 || !sum || !t_end || (ns && !s) || (ne && !e)) return -1;
  if (t_end[0] < c->t_prev) return -1;
  for (uint32_t w = 1; w < W; ++w) if (t_end[w] < t_end[w - 1]) return -1;

  const int64_t t_begin = c->t_prev;
  uint64_t *dropped = (uint64_t *)calloc(W, sizeof(uint64_t));
  int32_t *swin = (int32_t *)malloc(sizeof(int32_t) * (ns ? ns : 1));
  int32_t *ewin = (int32_t *)malloc(sizeof(int32_t) * (ne ? ne : 1));
  int rc = classify(1, s, ns, c, t_end, W, t_begin, swin, dropped);
  if (rc == 0) rc = classify(0, e, ne, c, t_end, W, t_begin, ewin, dropped);
  if (rc != 0) {
    free(dropped); free(swin); free(ewin);
    c->sticky = rc;
    return rc;
  }
  uint64_t *sstart = (uint64_t *)malloc(sizeof(uint64_t) * (W + 1));
  uint64_t *estart = (uint64_t *)malloc(sizeof(uint64_t) * (W + 1));
  uint64_t *sorder = (uint64_t *)malloc(sizeof(uint64_t) * (ns ? ns : 1));
  uint64_t *eorder = (uint64_t *)malloc(sizeof(uint64_t) * (ne ? ne : 1));
  bucket(swin, ns, W, sstart, sorder);
  bucket(ewin, ne, W, estart, eorder);

  const uint32_t nb = c->nb, nc = c->nc, nk = c->nk;
  uint16_t *L = (uint16_t *)malloc(sizeof(uint16_t) * nb);
  uint16_t *mx = (uint16_t *)malloc(sizeof(uint16_t) * nb);
  uint16_t *mn = (uint16_t *)malloc(sizeof(uint16_t) * nb);
  int64_t *t = (int64_t *)malloc(sizeof(int64_t) * nb);
  uint64_t *I = (uint64_t *)malloc(sizeof(uint64_t) * nb);
  uint32_t *cnt = (uint32_t *)malloc(sizeof(uint32_t) * nb);
  uint8_t *full = (uint8_t *)malloc(nb);
  uint8_t *active = (uint8_t *)malloc(nc);
  uint8_t *anyfull = (uint8_t *)malloc(nc);
  rank_item *items = (rank_item *)malloc(sizeof(rank_item) * nb);

  for (uint32_t w = 0; w < W; ++w) {
    const int64_t tp = (w == 0) ? t_begin : t_end[w - 1];
    const int64_t te = t_end[w];
    const int64_t Wlen = te - tp;
    orc_summary *S = &sum[w];
    memset(S, 0, sizeof(*S));
    S->t_begin = tp;
    S->t_end = te;
    S->n_dropped = dropped[w];
    S->n_samples = sstart[w + 1] - sstart[w];
    S->n_events = estart[w + 1] - estart[w];

    /* ---- buffer fold: L = level held since t, I accumulates level * dt (L181, L199) ---- */
    for (uint32_t b = 0; b < nb; ++b) {
      L[b] = c->lvl[b]; /* carry-in level counts toward max/min even if held for 0 ticks */
      t[b] = tp;
      I[b] = 0;
      mx[b] = L[b];
      mn[b] = L[b];
      cnt[b] = 0;
    }
    for (uint64_t q = sstart[w]; q < sstart[w + 1]; ++q) {
      const orc_sample *r = &s[sorder[q]]; /* ingest order: equal ts -> later record wins */
      uint32_t b = r->buffer_id;
      I[b] += (uint64_t)L[b] * (uint64_t)(r->ts - t[b]);
      t[b] = r->ts;
      L[b] = r->level;
      if (r->level > mx[b]) mx[b] = r->level;
      if (r->level < mn[b]) mn[b] = r->level;
      cnt[b]++;
    }
    uint64_t digest = 0;
    uint32_t touched = 0;
    for (uint32_t b = 0; b < nb; ++b) {
      I[b] += (uint64_t)L[b] * (uint64_t)(te - t[b]);
      /* held for the whole window, carry-in included: full (R9) or, in the paper's looser
       * reading, non-empty ("any content in a buffer", L229) */
      full[b] = c->hang_mode == 1 ? (mn[b] >= 1) : (mn[b] == c->cap[b]);
      c->lvl[b] = L[b];
      if (cnt[b] > 0) {
        touched++;
        digest += orc_digest_term(b, L[b], mx[b], mn[b], c->cap[b], cnt[b], (int64_t)I[b]);
      }
      if (all_stats || (last_stats && w == W - 1)) {
        orc_bstat st;
        memset(&st, 0, sizeof(st));
        st.integral = (int64_t)I[b];
        st.last = L[b];
        st.max = mx[b];
        st.min = mn[b];
        st.capacity = c->cap[b];
        st.n_samples = cnt[b];
        st.mean_occ = Wlen > 0 ? (double)(int64_t)I[b] / (double)((int64_t)c->cap[b] * Wlen) : 0.0;
        if (all_stats) all_stats[(uint64_t)w * nb + b] = st;
        if (last_stats && w == W - 1) last_stats[b] = st;
      }
    }
    S->digest = digest;
    S->n_touched = touched;

    /* ---- task events -> progress bars (L131) ---- */
    memset(active, 0, nc);
    for (uint64_t q = estart[w]; q < estart[w + 1]; ++q) {
      const orc_event *r = &e[eorder[q]];
      uint32_t comp = r->meta & 0xFFFFFu, kern = (r->meta >> 20) & 0x7FFu, kind = r->meta >> 31;
      if (kind == 0) { c->c_started[comp]++; c->k_started[kern]++; }
      else { c->c_ended[comp]++; c->k_ended[kern]++; }
      active[comp] = 1;
    }
    if (prog)
      for (uint32_t k = 0; k < nk; ++k) {
        orc_progress *P = &prog[(uint64_t)w * nk + k];
        if (!c->live[k]) { memset(P, 0, sizeof(*P)); continue; } /* free bar id: all zero */
        P->total = c->ktotal[k];
        P->started = c->k_started[k];
        P->finished = c->k_ended[k];
        P->in_flight = c->k_started[k] - c->k_ended[k];
        P->not_started = c->ktotal[k] - c->k_started[k];
      }

    /* ---- Bottleneck Analyzer list: rank every (owned) buffer by its last level ---- */
    if (topk || topk_n) {
      uint32_t m = 0;
      for (uint32_t b = 0; b < nb; ++b)
        if (c->owned[c->owner[b]]) {
          items[m].id = b; items[m].l = c->lvl[b]; items[m].c = c->cap[b]; items[m].I = I[b]; ++m;
        }
      qsort(items, m, sizeof(rank_item), c->rank_mode == 1 ? cmp_size : c->rank_mode == 2 ? cmp_mean : cmp_percent);
      uint32_t kk = c->k < m ? c->k : m;
      for (uint32_t i = 0; i < kk; ++i) c->persist[items[i].id]++;
      if (topk_n) topk_n[w] = kk;
      if (topk)
        for (uint32_t i = 0; i < c->k; ++i) {
          orc_topk *o = &topk[(uint64_t)w * c->k + i];
          if (i < kk) { o->buffer_id = items[i].id; o->level = items[i].l; o->capacity = items[i].c; }
          else { o->buffer_id = 0xFFFFFFFFu; o->level = 0; o->capacity = 0; }
        }
    }

    /* ---- hang flag (L227-L229): a buffer full all window and no task event, H windows ---- */
    memset(anyfull, 0, nc);
    for (uint32_t b = 0; b < nb; ++b) if (full[b]) anyfull[c->owner[b]] = 1;
    uint32_t nh = 0;
    for (uint32_t q = 0; q < nc; ++q) {
      int cond = anyfull[q] && !active[q];
      c->run[q] = cond ? c->run[q] + 1 : 0;
      int flagged = c->run[q] >= c->H;
      if (hung) hung[(uint64_t)w * nc + q] = (uint8_t)flagged;
      nh += (uint32_t)flagged;
    }
    S->n_hung = nh;
  }
  if (comps)
    for (uint32_t q = 0; q < nc; ++q) {
      comps[q].started = c->c_started[q];
      comps[q].finished = c->c_ended[q];
      comps[q].in_flight = c->c_started[q] - c->c_ended[q];
    }
  c->t_prev = t_end[W - 1];

  free(L); free(mx); free(mn); free(t); free(I); free(cnt); free(full); free(active); free(anyfull);
  free(items); free(dropped); free(swin); free(ewin); free(sstart); free(estart); free(sorder); free(eorder);
  return 0;
}

int orc_merge_topk(const orc_topk *const *shard_topk, const uint32_t *const *shard_n, uint32_t n_shards,
                   uint32_t W, uint32_t k, int32_t rank_mode, orc_topk *out, uint32_t *out_n) {
  rank_item *items = (rank_item *)malloc(sizeof(rank_item) * ((uint64_t)n_shards * k + 1));
  for (uint32_t w = 0; w < W; ++w) {
    uint32_t m = 0;
    for (uint32_t r = 0; r < n_shards; ++r)
      for (uint32_t i = 0; i < shard_n[r][w]; ++i) {
        const orc_topk *t = &shard_topk[r][(uint64_t)w * k + i];
        items[m].id = t->buffer_id; items[m].l = t->level; items[m].c = t->capacity; ++m;
      }
    qsort(items, m, sizeof(rank_item), rank_mode == 1 ? cmp_size : cmp_percent);
    uint32_t kk = k < m ? k : m;
    out_n[w] = kk;
    for (uint32_t i = 0; i < k; ++i) {
      orc_topk *o = &out[(uint64_t)w * k + i];
      if (i < kk) { o->buffer_id = items[i].id; o->level = items[i].l; o->capacity = items[i].c; }
      else { o->buffer_id = 0xFFFFFFFFu; o->level = 0; o->capacity = 0; }
    }
  }
  free(items);
  return 0;
}

/* Windows-in-top-k counter of every buffer since create / reset. */
void orc_persistence(const orc_ctx *c, uint32_t *out) {
  for (uint32_t b = 0; b < c->nb; ++b) out[b] = c->persist[b];
}

/* Progress bar registry (CreateProgressBar / UpdateProgressBar / DestroyProgressBar, L99, L131):
 * create takes the lowest free id and starts its counts at zero; update sets the total; destroy
 * frees the id (events naming a free id are field-invalid).  Return 0, or -1 (no free id /
 * id not live / out of range). */
int orc_bar_create(orc_ctx *c, int64_t total, uint32_t *id) {
  for (uint32_t k = 0; k < c->nk; ++k)
    if (!c->live[k]) {
      c->live[k] = 1;
      c->ktotal[k] = total;
      c->k_started[k] = c->k_ended[k] = 0;
      *id = k;
      return 0;
    }
  return -1;
}
int orc_bar_update(orc_ctx *c, uint32_t id, int64_t total) {
  if (id >= c->nk || !c->live[id]) return -1;
  c->ktotal[id] = total;
  return 0;
}
int orc_bar_destroy(orc_ctx *c, uint32_t id) {
  if (id >= c->nk || !c->live[id]) return -1;
  c->live[id] = 0;
  return 0;
}
