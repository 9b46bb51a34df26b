/*
 * gpa_mine_fimi -- mine a FIMI-format transaction file with libgpapriori (plain C, C ABI only).
 *
 *   usage: gpa_mine_fimi <file.dat> <minsup, e.g. 0.01> [max_k]
 *
 * Input: one transaction per line, whitespace-separated non-negative item ids (the FIMI
 * repository format the paper's datasets use, PAPER.md P18@3425).  Output: one frequent itemset
 * per line, "i1 i2 ... ik (support)", in canonical order (by k, then lexicographic), followed by
 * a per-generation summary on stderr.  minsup is a decimal ratio; the count threshold is
 * max(1, ceil(minsup * N)) computed exactly by gpa_min_count.
 */
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

#include "gpapriori.h"

static void die(const char* what, gpa_status st) {
  fprintf(stderr, "%s failed: status %d: %s\n", what, (int)st, gpa_last_error());
  exit(1);
}

/* decimal string -> num/den exactly (e.g. "0.005" -> 5/1000) */
static void parse_ratio(const char* s, uint64_t* num, uint64_t* den) {
  uint64_t n = 0, d = 1;
  int frac = 0;
  for (const char* p = s; *p; ++p) {
    if (*p == '.') { frac = 1; continue; }
    if (*p < '0' || *p > '9') { fprintf(stderr, "bad minsup '%s'\n", s); exit(1); }
    n = n * 10 + (uint64_t)(*p - '0');
    if (frac) d *= 10;
  }
  *num = n;
  *den = d;
}

int main(int argc, char** argv) {
  if (argc < 3) {
    fprintf(stderr, "usage: %s <file.dat> <minsup> [max_k]\n", argv[0]);
    return 2;
  }
  FILE* f = fopen(argv[1], "r");
  if (!f) { perror(argv[1]); return 1; }
  size_t cap_tx = 1024, cap_it = 1 << 16, n_tx = 0, nnz = 0;
  uint64_t* offsets = malloc(sizeof(uint64_t) * (cap_tx + 1));
  uint32_t* items = malloc(sizeof(uint32_t) * cap_it);
  uint32_t n_items = 0;
  char* line = NULL;
  size_t len = 0;
  offsets[0] = 0;
  while (getline(&line, &len, f) >= 0) {
    char* p = line;
    for (;;) {
      while (*p == ' ' || *p == '\t' || *p == '\r' || *p == '\n') ++p;
      if (!*p) break;
      char* end;
      unsigned long v = strtoul(p, &end, 10);
      if (end == p) { fprintf(stderr, "bad item in line %zu\n", n_tx + 1); return 1; }
      if (nnz == cap_it) { cap_it *= 2; items = realloc(items, sizeof(uint32_t) * cap_it); }
      items[nnz++] = (uint32_t)v;
      if (v + 1 > n_items) n_items = (uint32_t)(v + 1);
      p = end;
    }
    if (n_tx + 1 == cap_tx) { cap_tx *= 2; offsets = realloc(offsets, sizeof(uint64_t) * (cap_tx + 1)); }
    offsets[++n_tx] = nnz;
  }
  free(line);
  fclose(f);

  uint64_t num, den;
  parse_ratio(argv[2], &num, &den);
  const uint64_t min_count = gpa_min_count(n_tx, num, den);
  gpa_tx_csr db = {n_tx, offsets, items, n_items, GPA_MEM_HOST};
  gpa_options opt;
  gpa_options_default(&opt);
  if (argc > 3) opt.max_k = (uint32_t)atoi(argv[3]);
  gpa_result* res = NULL;
  gpa_status st = gpa_mine(&db, min_count, NULL, &opt, &res);
  if (st != GPA_OK) die("gpa_mine", st);

  uint64_t n_sets = 0;
  uint32_t max_k = 0, n_levels = 0;
  gpa_result_count(res, &n_sets, &max_k);
  for (uint64_t i = 0; i < n_sets; ++i) {
    const uint32_t* its;
    uint32_t k, sup;
    if ((st = gpa_result_get(res, i, &its, &k, &sup)) != GPA_OK) die("gpa_result_get", st);
    for (uint32_t j = 0; j < k; ++j) printf(j ? " %u" : "%u", its[j]);
    printf(" (%u)\n", sup);
  }
  gpa_result_n_levels(res, &n_levels);
  fprintf(stderr, "%s: N = %zu, items < %u, min_count = %llu, |F| = %llu, longest = %u\n", argv[1], n_tx, n_items,
          (unsigned long long)min_count, (unsigned long long)n_sets, max_k);
  for (uint32_t k = 1; k <= n_levels; ++k) {
    gpa_level_stats ls;
    gpa_result_level_stats(res, k, &ls);
    fprintf(stderr, "  k=%u |C|=%llu |L|=%llu count %.3f ms\n", k, (unsigned long long)ls.n_cand,
            (unsigned long long)ls.n_freq, ls.count_ms);
  }
  gpa_result_destroy(res);
  free(offsets);
  free(items);
  return 0;
}
