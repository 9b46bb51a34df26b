/*
 * gen/quest.c -- seeded synthetic transaction generators (test/bench input only).
 *
 * This module holds NO arithmetic of the mined method (no support counting, no
 * candidate generation, no thresholds): it only draws random transactions.  It is
 * shared by the oracle side and the CUDA side as the single source of inputs, as
 * the build rules allow.
 *
 * IBM-Quest-style market-basket generator after Agrawal & Srikant, VLDB 1994
 * (the paper's ref. [2], PAPER.md P28@1007): a pool of L "potentially large
 * itemsets" (patterns) with Poisson(I) sizes, exponentially distributed weights,
 * correlation between consecutive patterns and per-pattern corruption levels;
 * transactions of Poisson(T) size are filled with corrupted patterns.  The paper's
 * T40I10D100K dataset (Table 2, PAPER.md P23@308) is such a file; the FIMI
 * originals are not available offline, so we regenerate the shape.
 *
 * Determinism: splitmix64 seeding + xoshiro256**.  Patterns depend only on the
 * base seed; transactions are produced in chunks of GEN_CHUNK transactions, each
 * chunk seeded with splitmix64(seed, chunk index) and starting with empty carry-over
 * state, so any contiguous chunk range (one rank's shard) can be generated alone and
 * the concatenation is identical for any partition.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <math.h>
#include <pthread.h>

#define GEN_CHUNK 102400u /* 200 x 512 transactions: rank shards stay 512-aligned */

typedef struct { uint64_t s[4]; } rng_t;

static uint64_t splitmix64(uint64_t* x) {
  uint64_t z = (*x += 0x9E3779B97F4A7C15ull);
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}
static void rng_seed(rng_t* r, uint64_t seed, uint64_t stream) {
  uint64_t x = seed * 0x9E3779B97F4A7C15ull ^ (stream + 0x632BE59BD9B4E019ull);
  for (int i = 0; i < 4; ++i) r->s[i] = splitmix64(&x);
}
static inline uint64_t rotl(uint64_t x, int k) { return (x << k) | (x >> (64 - k)); }
static inline uint64_t rng_next(rng_t* r) {
  uint64_t* s = r->s;
  uint64_t res = rotl(s[1] * 5, 7) * 9, t = s[1] << 17;
  s[2] ^= s[0]; s[3] ^= s[1]; s[1] ^= s[2]; s[0] ^= s[3]; s[2] ^= t; s[3] = rotl(s[3], 45);
  return res;
}
static inline double rng_u01(rng_t* r) { return (rng_next(r) >> 11) * (1.0 / 9007199254740992.0); }
static inline uint32_t rng_below(rng_t* r, uint32_t n) { return (uint32_t)(((unsigned __int128)rng_next(r) * n) >> 64); }
static uint32_t rng_poisson(rng_t* r, double lam) {
  /* Knuth's product method; lam <= ~60 here so exp(-lam) is well inside double range. */
  double L = exp(-lam), p = 1.0; uint32_t k = 0;
  do { ++k; p *= rng_u01(r); } while (p > L);
  return k - 1;
}
static double rng_exp(rng_t* r, double mean) { return -mean * log(1.0 - rng_u01(r)); }
static double rng_normal(rng_t* r, double mu, double sd) {
  double u1 = 1.0 - rng_u01(r), u2 = rng_u01(r);
  return mu + sd * sqrt(-2.0 * log(u1)) * cos(6.283185307179586 * u2);
}

typedef struct {
  uint32_t n_items, n_pat;
  uint32_t* pat_off;   /* n_pat+1 */
  uint32_t* pat_items; /* concatenated, distinct within a pattern */
  double* cum_w;       /* cumulative normalised weights, n_pat */
  double* corrupt;     /* per-pattern corruption level in [0,1] */
  double avg_len;
} quest_model;

static int u32_cmp(const void* a, const void* b) {
  uint32_t x = *(const uint32_t*)a, y = *(const uint32_t*)b; return (x > y) - (x < y);
}

static int in_list(const uint32_t* v, uint32_t n, uint32_t x) {
  for (uint32_t i = 0; i < n; ++i) if (v[i] == x) return 1;
  return 0;
}

static void quest_build(quest_model* m, uint64_t seed, uint32_t n_items, uint32_t n_pat, double avg_pat, double corr) {
  rng_t r; rng_seed(&r, seed, 0xA11CEull);
  m->n_items = n_items; m->n_pat = n_pat;
  m->pat_off = (uint32_t*)malloc((n_pat + 1) * sizeof(uint32_t));
  uint32_t cap = n_pat * (uint32_t)(avg_pat * 3 + 8);
  m->pat_items = (uint32_t*)malloc(cap * sizeof(uint32_t));
  m->cum_w = (double*)malloc(n_pat * sizeof(double));
  m->corrupt = (double*)malloc(n_pat * sizeof(double));
  uint32_t pos = 0; double wsum = 0;
  m->pat_off[0] = 0;
  for (uint32_t p = 0; p < n_pat; ++p) {
    uint32_t sz = rng_poisson(&r, avg_pat);
    if (sz < 1) sz = 1;
    if (sz > n_items) sz = n_items;
    if (pos + sz > cap) { cap = 2 * (pos + sz); m->pat_items = (uint32_t*)realloc(m->pat_items, cap * sizeof(uint32_t)); }
    uint32_t* cur = m->pat_items + pos, n = 0;
    if (p > 0) { /* correlation: an exponentially distributed fraction comes from the previous pattern */
      double frac = rng_exp(&r, corr); if (frac > 1.0) frac = 1.0;
      uint32_t* prev = m->pat_items + m->pat_off[p - 1];
      uint32_t np = m->pat_off[p] - m->pat_off[p - 1];
      uint32_t take = (uint32_t)(frac * sz + 0.5); if (take > np) take = np;
      for (uint32_t t = 0; t < take && n < sz; ++t) {
        uint32_t x = prev[rng_below(&r, np)];
        if (!in_list(cur, n, x)) cur[n++] = x;
      }
    }
    while (n < sz) { uint32_t x = rng_below(&r, n_items); if (!in_list(cur, n, x)) cur[n++] = x; }
    pos += n; m->pat_off[p + 1] = pos;
    double w = rng_exp(&r, 1.0); wsum += w; m->cum_w[p] = wsum;
    double c = rng_normal(&r, 0.5, 0.1); m->corrupt[p] = c < 0 ? 0 : (c > 1 ? 1 : c);
  }
  for (uint32_t p = 0; p < n_pat; ++p) m->cum_w[p] /= wsum;
  m->cum_w[n_pat - 1] = 1.0;
}
static void quest_free(quest_model* m) { free(m->pat_off); free(m->pat_items); free(m->cum_w); free(m->corrupt); }

static uint32_t pick_pattern(const quest_model* m, rng_t* r) {
  double u = rng_u01(r); uint32_t lo = 0, hi = m->n_pat - 1;
  while (lo < hi) { uint32_t mid = (lo + hi) / 2; if (m->cum_w[mid] < u) lo = mid + 1; else hi = mid; }
  return lo;
}

/* Generate transactions [c*GEN_CHUNK, min(n_tx,(c+1)*GEN_CHUNK)) of chunk c into a growable buffer. */
typedef struct { uint32_t* items; uint64_t n, cap; uint32_t* lens; } chunk_out;

static void push_item(chunk_out* o, uint32_t x) {
  if (o->n == o->cap) { o->cap = o->cap ? 2 * o->cap : 1 << 16; o->items = (uint32_t*)realloc(o->items, o->cap * 4); }
  o->items[o->n++] = x;
}

static void quest_chunk(const quest_model* m, uint64_t seed, uint64_t chunk, uint32_t n_in_chunk, double avg_tx, chunk_out* o) {
  rng_t r; rng_seed(&r, seed, 0x100000ull + chunk);
  uint32_t* tmp = (uint32_t*)malloc(sizeof(uint32_t) * (m->n_items + 64));
  uint32_t* pat = (uint32_t*)malloc(sizeof(uint32_t) * (m->n_items + 64));
  uint32_t carry_n = 0; uint32_t* carry = (uint32_t*)malloc(sizeof(uint32_t) * (m->n_items + 64));
  o->lens = (uint32_t*)malloc(sizeof(uint32_t) * (n_in_chunk ? n_in_chunk : 1));
  for (uint32_t t = 0; t < n_in_chunk; ++t) {
    uint32_t target = rng_poisson(&r, avg_tx);
    if (target < 1) target = 1;
    uint32_t len = 0;
    if (carry_n) { memcpy(tmp, carry, carry_n * 4); len = carry_n; carry_n = 0; }
    int guard = 0;
    while (len < target && guard++ < 1000) {
      uint32_t p = pick_pattern(m, &r);
      const uint32_t* src = m->pat_items + m->pat_off[p];
      uint32_t np = m->pat_off[p + 1] - m->pat_off[p];
      memcpy(pat, src, np * 4);
      /* corruption: keep dropping a random item while u < c_p */
      while (np > 0 && rng_u01(&r) < m->corrupt[p]) { uint32_t j = rng_below(&r, np); pat[j] = pat[--np]; }
      if (np == 0) continue;
      if (len + np > target && len > 0) {
        if (rng_u01(&r) < 0.5) { memcpy(tmp + len, pat, np * 4); len += np; }
        else { memcpy(carry, pat, np * 4); carry_n = np; }
        break;
      }
      memcpy(tmp + len, pat, np * 4); len += np;
      if (len > m->n_items) break;
    }
    qsort(tmp, len, 4, u32_cmp);
    uint32_t u = 0;
    for (uint32_t i = 0; i < len; ++i) if (u == 0 || tmp[i] != tmp[u - 1]) tmp[u++] = tmp[i];
    for (uint32_t i = 0; i < u; ++i) push_item(o, tmp[i]);
    o->lens[t] = u;
  }
  free(tmp); free(pat); free(carry);
}

typedef struct {
  const quest_model* m; uint64_t seed, n_tx; double avg_tx;
  uint64_t c0, c1; chunk_out* outs; int tid, nth;
} job_t;

static void* worker(void* arg) {
  job_t* j = (job_t*)arg;
  for (uint64_t c = j->c0 + j->tid; c < j->c1; c += j->nth) {
    uint64_t start = c * GEN_CHUNK, end = start + GEN_CHUNK; if (end > j->n_tx) end = j->n_tx;
    quest_chunk(j->m, j->seed, c, (uint32_t)(end - start), j->avg_tx, &j->outs[c - j->c0]);
  }
  return NULL;
}

uint32_t gen_chunk_size(void) { return GEN_CHUNK; }

/*
 * Generate transactions [tx_begin, tx_end) of the Quest dataset (n_tx total; tx_begin must be a
 * multiple of GEN_CHUNK).  On success returns 0 and library-allocated arrays *offsets_out
 * (tx_end-tx_begin+1 entries, starting at 0) and *items_out (*nnz_out entries); release them
 * with gen_free().  Each transaction is sorted and duplicate-free.
 */
int gen_quest(uint64_t seed, uint64_t n_tx, double avg_tx, double avg_pat, uint32_t n_items, uint32_t n_pat,
              double corr, uint64_t tx_begin, uint64_t tx_end, int n_threads,
              uint64_t** offsets_out, uint32_t** items_out, uint64_t* nnz_out) {
  if (tx_begin % GEN_CHUNK || tx_end > n_tx || tx_begin > tx_end || n_items == 0 || n_pat == 0) return 1;
  quest_model m; quest_build(&m, seed, n_items, n_pat, avg_pat, corr);
  uint64_t c0 = tx_begin / GEN_CHUNK, c1 = (tx_end + GEN_CHUNK - 1) / GEN_CHUNK;
  uint64_t nc = c1 - c0;
  chunk_out* outs = (chunk_out*)calloc(nc ? nc : 1, sizeof(chunk_out));
  if (n_threads < 1) n_threads = 1;
  pthread_t* th = (pthread_t*)malloc(sizeof(pthread_t) * n_threads);
  job_t* jobs = (job_t*)malloc(sizeof(job_t) * n_threads);
  for (int t = 0; t < n_threads; ++t) {
    jobs[t] = (job_t){&m, seed, n_tx, avg_tx, c0, c1, outs, t, n_threads};
    pthread_create(&th[t], NULL, worker, &jobs[t]);
  }
  for (int t = 0; t < n_threads; ++t) pthread_join(th[t], NULL);
  /* assemble [tx_begin, tx_end) (the last chunk may extend beyond tx_end: truncate) */
  uint64_t total = 0;
  for (uint64_t c = c0; c < c1; ++c) total += outs[c - c0].n;
  uint64_t* offsets = (uint64_t*)malloc(sizeof(uint64_t) * (tx_end - tx_begin + 1));
  uint32_t* items = (uint32_t*)malloc(sizeof(uint32_t) * (total ? total : 1));
  uint64_t nnz = 0, k = 0;
  offsets[0] = 0;
  for (uint64_t c = c0; c < c1; ++c) {
    chunk_out* o = &outs[c - c0];
    uint64_t start = c * GEN_CHUNK, end = start + GEN_CHUNK; if (end > n_tx) end = n_tx;
    uint64_t take_end = end < tx_end ? end : tx_end, pos = 0;
    for (uint64_t t = start; t < take_end; ++t) {
      uint32_t len = o->lens[t - start];
      memcpy(items + nnz, o->items + pos, (size_t)len * 4);
      pos += len; nnz += len; ++k;
      offsets[k] = nnz;
    }
    free(o->items); free(o->lens);
  }
  *offsets_out = offsets; *items_out = items; *nnz_out = nnz;
  free(outs); free(th); free(jobs); quest_free(&m);
  return 0;
}

void gen_free(void* p) { free(p); }
