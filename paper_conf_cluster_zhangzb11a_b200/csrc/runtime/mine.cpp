// Level-wise mining (gpa_mine) and its result object.
//
// The loop is the paper's Apriori (PAPER.md P13@338-652) with the GPU doing support counting
// (P2@505, P18@394): generation 1 by the device histogram, the static bitset of the frequent
// items (P18@755), then per generation k >= 2: candidates C_k (k = 2: every pair of rows,
// counted by the tiled pair kernel; k >= 3: join + prune of L_{k-1} grouped by prefix),
// counts on the GPU (+ NCCL all-reduce across ranks), counts back to the host ("the support
// value results are copied back to main memory", P18@672), L_k = { c : count >= min_count }
// (P13@474, ">=" per DESIGN.md Q1).  Stops when L_k or C_{k+1} is empty (P13@652).
#include <algorithm>
#include <chrono>

#include "internal.h"
#include "pool.h"

struct gpa_level_data {
  uint32_t k = 0;
  uint64_t n_cand = 0, n_freq = 0, n_groups = 0;
  std::vector<uint32_t> freq_items;    // n_freq * k, original ids, lexicographic
  std::vector<uint32_t> freq_support;  // n_freq
  std::vector<uint32_t> cand_items;    // n_cand * k (GPA_KEEP_CANDIDATES)
  std::vector<uint32_t> cand_counts;   // n_cand     (GPA_KEEP_CANDIDATES)
  bool kept = false;
  gpa_level_stats stats{};
};

struct gpa_result {
  uint64_t n_tx = 0, min_count = 0;
  uint32_t n_items = 0;
  std::vector<gpa_level_data> levels;  // levels[0] is k = 1
  std::vector<uint64_t> freq_start;    // prefix sums of n_freq
  double phase_ms[GPA_PHASE_COUNT_] = {0};
};

namespace gpa {
namespace {

double now_ms() {
  return std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now().time_since_epoch()).count();
}

// Record generation k.  Candidates are the grouped batch b (k >= 3) or, for k = 2 (b == nullptr),
// all pairs of the n rows in lexicographic order.  Returns L_k in row ids (lexicographic).
// Two parallel passes over contiguous candidate ranges: count the frequent candidates of each
// range, then write L_k, the frequent itemsets (original ids) and their supports at exact
// offsets (no growing vectors, no concatenation).
std::vector<uint32_t> record_level(gpa_result* R, const gpa_bitset* bs, uint32_t k, const GroupedBatch* b, uint64_t M,
                                   const std::vector<uint32_t>& counts, bool keep, uint64_t* n_freq) {
  gpa_level_data lv;
  lv.k = k;
  lv.n_cand = M;
  lv.kept = keep;
  const auto& ior = bs->item_of_row;
  const uint32_t theta = (uint32_t)R->min_count;
  const uint64_t n = bs->n_rows;
  // outer units: groups (k >= 3) or first items a (k = 2)
  const uint64_t U = b ? b->groups() : (n ? n - 1 : 0);
  auto unit_begin = [&](uint64_t u) -> uint64_t { return b ? b->ext_off[u] : pair_index(u, u + 1, n); };
  if (keep) {
    lv.cand_items.resize(M * k);
    lv.cand_counts = counts;
  }
  const size_t T = std::min<size_t>(pool_threads() * 4, std::max<uint64_t>(1, M / 4096));
  std::vector<uint64_t> ucut(T + 1, U);
  ucut[0] = 0;
  for (size_t t = 1; t < T; ++t) {  // equal candidate counts per range
    const uint64_t target = M * t / T;
    uint64_t lo = ucut[t - 1], hi = U;
    while (lo < hi) {
      const uint64_t mid = (lo + hi) / 2;
      if (unit_begin(mid) < target) lo = mid + 1; else hi = mid;
    }
    ucut[t] = lo;
  }
  std::vector<uint64_t> nf(T + 1, 0);
  parallel_for(T, [&](size_t t) {
    const uint64_t c0 = ucut[t] < U ? unit_begin(ucut[t]) : M, c1 = ucut[t + 1] < U ? unit_begin(ucut[t + 1]) : M;
    uint64_t c = 0;
    for (uint64_t m = c0; m < c1; ++m) c += counts[m] >= theta;
    nf[t + 1] = c;
  });
  for (size_t t = 0; t < T; ++t) nf[t + 1] += nf[t];
  const uint64_t F = nf[T];
  std::vector<uint32_t> Lk(F * k);
  lv.freq_items.resize(F * k);
  lv.freq_support.resize(F);
  parallel_for(T, [&](size_t t) {
    uint64_t f = nf[t];
    auto emit = [&](uint64_t m, const uint32_t* pre, uint32_t last) {
      if (keep) {
        uint32_t* dst = lv.cand_items.data() + m * k;
        for (uint32_t j = 0; j + 1 < k; ++j) dst[j] = ior[pre[j]];
        dst[k - 1] = ior[last];
      }
      if (counts[m] >= theta) {
        uint32_t* lrow = Lk.data() + f * k;
        uint32_t* irow = lv.freq_items.data() + f * k;
        for (uint32_t j = 0; j + 1 < k; ++j) {
          lrow[j] = pre[j];
          irow[j] = ior[pre[j]];
        }
        lrow[k - 1] = last;
        irow[k - 1] = ior[last];
        lv.freq_support[f] = counts[m];
        ++f;
      }
    };
    for (uint64_t u = ucut[t]; u < ucut[t + 1]; ++u) {
      if (b) {
        for (uint64_t j = b->ext_off[u]; j < b->ext_off[u + 1]; ++j) emit(j, b->prefix.data() + u * (k - 1), b->ext[j]);
      } else {
        const uint32_t a = (uint32_t)u;
        uint64_t m = unit_begin(u);
        for (uint32_t c = a + 1; c < n; ++c, ++m) emit(m, &a, c);
      }
    }
  });
  lv.n_freq = F;
  *n_freq = F;
  R->levels.push_back(std::move(lv));
  return Lk;
}

}  // namespace

gpa_result* mine(const gpa_tx_csr* db, uint64_t min_count, const gpa_dist* dist, const gpa_options* opt_in) {
  const double t_start = now_ms();
  gpa_options opt;
  gpa_options_default(&opt);
  if (opt_in) opt = *opt_in;
  GPA_REQUIRE(min_count >= 1, GPA_ERR_INVALID, "min_count must be >= 1");
  const bool keep = (opt.flags & GPA_KEEP_CANDIDATES) != 0;
  const uint32_t max_k = opt.max_k ? opt.max_k : GPA_MAX_K;
  GPA_REQUIRE(min_count < (1ull << 32), GPA_ERR_INVALID, "min_count must be < 2^32");

  gpa_bitset* bs = bitset_build(db, min_count, dist, &opt);
  struct BsGuard {
    gpa_bitset* b;
    ~BsGuard() { bitset_free(b); }
  } bs_guard{bs};
  auto* R = new gpa_result();
  struct RGuard {
    gpa_result* r;
    ~RGuard() { delete r; }
  } r_guard{R};
  R->n_tx = bs->n_tx_global;
  R->min_count = min_count;
  R->n_items = bs->n_items;
  R->phase_ms[GPA_PHASE_UPLOAD] = bs->build_ms[0];
  R->phase_ms[GPA_PHASE_HISTOGRAM] = bs->build_ms[1];
  R->phase_ms[GPA_PHASE_BITSET] = bs->build_ms[2];
  cudaStream_t s = bs->stream;

  // generation 1: C_1 = all item ids, counts = the global histogram
  {
    gpa_level_data l1;
    l1.k = 1;
    l1.n_cand = bs->n_items;
    l1.kept = keep;
    if (keep) {
      l1.cand_items.resize(bs->n_items);
      for (uint32_t i = 0; i < bs->n_items; ++i) l1.cand_items[i] = i;
      l1.cand_counts = bs->item_counts;
    }
    for (uint32_t i = 0; i < bs->n_items; ++i)
      if (bs->item_counts[i] >= min_count) {
        l1.freq_items.push_back(i);
        l1.freq_support.push_back(bs->item_counts[i]);
      }
    l1.n_freq = l1.freq_items.size();
    l1.stats.n_cand = l1.n_cand;
    l1.stats.n_freq = l1.n_freq;
    R->levels.push_back(std::move(l1));
  }

  std::vector<uint32_t> L;  // L_{k-1} in row ids
  uint64_t nL = bs->n_rows;
  for (uint32_t r = 0; r < bs->n_rows; ++r) L.push_back(r);

  for (uint32_t k = 2; k <= max_k && nL > 0; ++k) {
    double t0 = now_ms();
    CountStats cs;
    GroupedBatch batch;
    uint64_t M = 0, G = 0;
    if (k == 2) {
      M = (uint64_t)bs->n_rows * (bs->n_rows - 1) / 2;
      G = bs->n_rows ? bs->n_rows - 1 : 0;
    } else {
      batch = candgen_join_prune(L, nL, k - 1);
      M = batch.size();
      G = batch.groups();
    }
    double t1 = now_ms();
    R->phase_ms[GPA_PHASE_CANDGEN] += t1 - t0;
    if (M == 0) break;
    if (k == 2) count_all_pairs(bs, opt.count_kernel, &cs);
    else count_grouped(bs, batch, opt.count_kernel, &cs);
    std::vector<uint32_t> counts(M);
    GPA_CUDA(cudaMemcpyAsync(counts.data(), bs->d_counts.p, M * sizeof(uint32_t), cudaMemcpyDeviceToHost, s));
    GPA_CUDA(cudaStreamSynchronize(s));
    double t2 = now_ms();
    R->phase_ms[GPA_PHASE_COUNT] += t2 - t1;

    uint64_t n_freq = 0;
    const double tr0 = now_ms();
    L = record_level(R, bs, k, k > 2 ? &batch : nullptr, M, counts, keep, &n_freq);
    if (trace_enabled())
      fprintf(stderr, "[gpa] k=%u M=%llu G=%llu: candgen %.2f ms, count phase %.2f ms (kernel %.2f), "
              "threshold %.2f ms -> |L|=%llu\n", k, (unsigned long long)M, (unsigned long long)G, t1 - t0, t2 - t1,
              cs.count_ms, now_ms() - tr0, (unsigned long long)n_freq);
    nL = n_freq;
    gpa_level_stats& st = R->levels.back().stats;
    st.n_cand = M;
    st.n_freq = n_freq;
    st.n_groups = G;
    st.kernel = cs.kernel;
    st.launches = cs.launches;
    st.count_ms = cs.count_ms;
    st.allreduce_ms = cs.allreduce_ms;
    st.candgen_ms = t1 - t0;
    R->phase_ms[GPA_PHASE_THRESHOLD] += now_ms() - t2;
  }

  uint64_t acc = 0;
  for (auto& lv : R->levels) {
    R->freq_start.push_back(acc);
    acc += lv.n_freq;
  }
  R->freq_start.push_back(acc);
  R->phase_ms[GPA_PHASE_TOTAL] = now_ms() - t_start;
  r_guard.r = nullptr;
  return R;
}

}  // namespace gpa

// ---------------------------------------------------------------- C ABI: mine + result

extern "C" gpa_status gpa_mine(const gpa_tx_csr* db, uint64_t min_count, const gpa_dist* dist, const gpa_options* opt,
                               gpa_result** out) {
  return gpa::guard([&] {
    GPA_REQUIRE(out, GPA_ERR_INVALID, "out is NULL");
    *out = gpa::mine(db, min_count, dist, opt);
  });
}

extern "C" gpa_status gpa_result_info(const gpa_result* r, uint64_t* n_tx, uint64_t* min_count) {
  return gpa::guard([&] {
    GPA_REQUIRE(r, GPA_ERR_INVALID, "result is NULL");
    if (n_tx) *n_tx = r->n_tx;
    if (min_count) *min_count = r->min_count;
  });
}

extern "C" gpa_status gpa_result_count(const gpa_result* r, uint64_t* n_itemsets, uint32_t* max_k) {
  return gpa::guard([&] {
    GPA_REQUIRE(r, GPA_ERR_INVALID, "result is NULL");
    if (n_itemsets) *n_itemsets = r->freq_start.back();
    if (max_k) {
      uint32_t m = 0;
      for (auto& lv : r->levels)
        if (lv.n_freq) m = lv.k;
      *max_k = m;
    }
  });
}

extern "C" gpa_status gpa_result_get(const gpa_result* r, uint64_t i, const uint32_t** items, uint32_t* k,
                                     uint32_t* support) {
  return gpa::guard([&] {
    GPA_REQUIRE(r, GPA_ERR_INVALID, "result is NULL");
    GPA_REQUIRE(i < r->freq_start.back(), GPA_ERR_RANGE, "index %llu out of range", (unsigned long long)i);
    size_t lvi = std::upper_bound(r->freq_start.begin(), r->freq_start.end(), i) - r->freq_start.begin() - 1;
    const gpa_level_data& lv = r->levels[lvi];
    const uint64_t j = i - r->freq_start[lvi];
    if (items) *items = lv.freq_items.data() + j * lv.k;
    if (k) *k = lv.k;
    if (support) *support = lv.freq_support[j];
  });
}

extern "C" gpa_status gpa_result_frequent(const gpa_result* r, uint32_t k, uint64_t* n, const uint32_t** items,
                                          const uint32_t** supports) {
  return gpa::guard([&] {
    GPA_REQUIRE(r, GPA_ERR_INVALID, "result is NULL");
    GPA_REQUIRE(k >= 1, GPA_ERR_INVALID, "k must be >= 1");
    if (k > r->levels.size()) {
      if (n) *n = 0;
      if (items) *items = nullptr;
      if (supports) *supports = nullptr;
      return;
    }
    const gpa_level_data& lv = r->levels[k - 1];
    if (n) *n = lv.n_freq;
    if (items) *items = lv.freq_items.data();
    if (supports) *supports = lv.freq_support.data();
  });
}

extern "C" gpa_status gpa_result_level(const gpa_result* r, uint32_t k, uint64_t* n_cand, uint64_t* n_freq,
                                       const uint32_t** cand, const uint32_t** counts) {
  return gpa::guard([&] {
    GPA_REQUIRE(r, GPA_ERR_INVALID, "result is NULL");
    GPA_REQUIRE(k >= 1 && k <= r->levels.size(), GPA_ERR_RANGE, "generation %u was not reached", k);
    const gpa_level_data& lv = r->levels[k - 1];
    if (n_cand) *n_cand = lv.n_cand;
    if (n_freq) *n_freq = lv.n_freq;
    if (cand) *cand = lv.kept ? lv.cand_items.data() : nullptr;
    if (counts) *counts = lv.kept ? lv.cand_counts.data() : nullptr;
  });
}

extern "C" gpa_status gpa_result_n_levels(const gpa_result* r, uint32_t* n_levels) {
  return gpa::guard([&] {
    GPA_REQUIRE(r && n_levels, GPA_ERR_INVALID, "NULL argument");
    *n_levels = (uint32_t)r->levels.size();
  });
}

extern "C" gpa_status gpa_result_level_stats(const gpa_result* r, uint32_t k, gpa_level_stats* out) {
  return gpa::guard([&] {
    GPA_REQUIRE(r && out, GPA_ERR_INVALID, "NULL argument");
    GPA_REQUIRE(k >= 1 && k <= r->levels.size(), GPA_ERR_RANGE, "generation %u was not reached", k);
    *out = r->levels[k - 1].stats;
  });
}

extern "C" gpa_status gpa_result_timing(const gpa_result* r, double ms_by_phase[GPA_PHASE_COUNT_]) {
  return gpa::guard([&] {
    GPA_REQUIRE(r && ms_by_phase, GPA_ERR_INVALID, "NULL argument");
    for (int i = 0; i < GPA_PHASE_COUNT_; ++i) ms_by_phase[i] = r->phase_ms[i];
  });
}

extern "C" gpa_status gpa_result_destroy(gpa_result* r) {
  return gpa::guard([&] { delete r; });
}

extern "C" const char* gpa_last_error(void) { return gpa::last_error_cstr(); }

extern "C" const char* gpa_version(void) { return "gpapriori-b200 0.1 sm_100a"; }
