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
#include <array>
#include <map>
#include <memory>
#include <mutex>
#include <chrono>
#include <cstdlib>
#include <cstring>
#include <deque>
#include <string>

#include "internal.h"
#include "pool.h"

// Allocator whose resize() leaves new elements uninitialised: F (tens of MB) is filled by parallel
// copies right after the resize, so a zero-fill would be a serial pass (and every page fault on a
// single thread) for nothing.
template <class T>
struct DefaultInitAlloc : std::allocator<T> {
  template <class U>
  struct rebind {
    using other = DefaultInitAlloc<U>;
  };
  DefaultInitAlloc() = default;
  template <class U>
  DefaultInitAlloc(const DefaultInitAlloc<U>&) noexcept {}
  template <class U>
  void construct(U* p) noexcept {
    ::new (static_cast<void*>(p)) U;
  }
  template <class U, class... A>
  void construct(U* p, A&&... a) {
    ::new (static_cast<void*>(p)) U(std::forward<A>(a)...);
  }
};
using FVec = std::vector<uint32_t, DefaultInitAlloc<uint32_t>>;

namespace gpa {
// Page-locked blocks that a result owns: the frequent itemsets of a generation are copied from the
// device straight into one (no host copy at the end of the loop), and a destroyed result returns
// its blocks here for the next call (cudaHostAlloc costs ~1 ms per MB-sized block).
struct PinnedCache {
  std::mutex mu;
  std::multimap<size_t, void*> free;
  void* get(size_t& bytes) {
    bytes = (bytes + (size_t(1) << 16) - 1) & ~((size_t(1) << 16) - 1);
    {
      std::lock_guard<std::mutex> lk(mu);
      auto it = free.lower_bound(bytes);
      if (it != free.end() && it->first <= 4 * bytes + (size_t(1) << 20)) {
        void* p = it->second;
        bytes = it->first;
        free.erase(it);
        return p;
      }
    }
    void* p = nullptr;
    GPA_CUDA(cudaHostAlloc(&p, bytes, cudaHostAllocDefault));
    return p;
  }
  void put(void* p, size_t bytes) {
    std::lock_guard<std::mutex> lk(mu);
    free.emplace(bytes, p);
  }
};
inline PinnedCache& pinned_cache() {
  static PinnedCache* c = new PinnedCache();   // never destroyed: results may outlive static teardown
  return *c;
}
}  // namespace gpa

struct gpa_level_data {
  uint32_t k = 0;
  uint64_t n_cand = 0, n_freq = 0, n_groups = 0;
  FVec freq_items;                     // n_freq * k, original ids, lexicographic (or in fi)
  FVec freq_support;                   // n_freq (or in fs)
  const uint32_t* fi = nullptr;        // when set: F in a page-locked block of the result
  const uint32_t* fs = nullptr;
  const uint32_t* items() const { return fi ? fi : freq_items.data(); }
  const uint32_t* supports() const { return fs ? fs : freq_support.data(); }
  std::vector<uint32_t> cand_items;    // n_cand * k (GPA_KEEP_CANDIDATES)
  std::vector<uint32_t> cand_counts;   // n_cand     (GPA_KEEP_CANDIDATES)
  bool kept = false;
  gpa_level_stats stats{};
};

struct gpa_result {
  uint64_t n_tx = 0, min_count = 0;
  uint32_t n_items = 0;
  std::vector<std::pair<void*, size_t>> pinned;   // page-locked blocks holding F (pinned_cache)
  gpa_result() = default;
  gpa_result(const gpa_result&) = delete;
  gpa_result& operator=(const gpa_result&) = delete;
  ~gpa_result() {
    for (auto& b : pinned) gpa::pinned_cache().put(b.first, b.second);
  }
  std::vector<gpa_level_data> levels;  // levels[0] is k = 1
  std::vector<uint64_t> freq_start;    // prefix sums of n_freq
  double phase_ms[GPA_PHASE_COUNT_] = {0};
};

namespace gpa {
namespace {

double now_ms() {
  return std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now().time_since_epoch()).count();
}

// GPA_HOST_TRACE=1: host timestamps of the level loop (no CUDA calls), printed after the loop
struct HostTrace {
  bool on = [] {
    const char* e = std::getenv("GPA_HOST_TRACE");
    return e && *e && *e != '0';
  }();
  std::vector<std::pair<std::string, double>> v;
  void mark(const char* what, uint32_t k) {
    if (on) v.emplace_back(std::string(what) + " k=" + std::to_string(k), now_ms());
  }
  void print() const {
    if (!on || v.empty()) return;
    for (size_t i = 0; i < v.size(); ++i)
      fprintf(stderr, "[gpa-host] %9.3f (+%7.3f) %s\n", v[i].second - v[0].second,
              i ? v[i].second - v[i - 1].second : 0.0, v[i].first.c_str());
  }
};

// Record generation k from the device-side threshold: L_k (F rows of k row ids, lexicographic)
// and supports come back from the GPU; they are mapped to original item ids in parallel.  With
// GPA_KEEP_CANDIDATES the whole C_k (the host batch b, or all pairs for k = 2) and its counts
// are recorded as well.
void record_level(gpa_result* R, const gpa_bitset* bs, uint32_t k, const GroupedBatch* b, uint64_t M,
                  FVec&& Litems, FVec&& Lsup, bool keep,
                  const std::vector<uint32_t>* counts) {
  gpa_level_data lv;
  lv.k = k;
  lv.n_cand = M;
  lv.kept = keep;
  const auto& ior = bs->item_of_row;
  const uint64_t F = Lsup.size();
  lv.freq_items = std::move(Litems);   // already mapped to original item ids on the device
  lv.freq_support = std::move(Lsup);
  if (keep) {
    lv.cand_counts = *counts;
    lv.cand_items.resize(M * k);
    if (b) {
      const uint64_t G = b->groups();
      parallel_for(std::min<size_t>(pool_threads() * 2, std::max<uint64_t>(1, G / 1024)), [&](size_t t) {
        const size_t TT = std::min<size_t>(pool_threads() * 2, std::max<uint64_t>(1, G / 1024));
        for (uint64_t g = G * t / TT; g < G * (t + 1) / TT; ++g)
          for (uint64_t j = b->ext_off[g]; j < b->ext_off[g + 1]; ++j) {
            uint32_t* dst = lv.cand_items.data() + j * k;
            for (uint32_t d = 0; d + 1 < k; ++d) dst[d] = ior[b->prefix[g * (k - 1) + d]];
            dst[k - 1] = ior[b->ext[j]];
          }
      });
    } else {   // generation 2: every pair of L_1 rows
      const uint64_t n = l1_size(bs);
      auto item = [&](uint64_t i) { return ior[bs->l1_sub ? bs->l1[i] : i]; };
      uint64_t m = 0;
      for (uint64_t a = 0; a + 1 < n; ++a)
        for (uint64_t c = a + 1; c < n; ++c, ++m) {
          lv.cand_items[2 * m] = item(a);
          lv.cand_items[2 * m + 1] = item(c);
        }
    }
  }
  lv.n_freq = F;
  R->levels.push_back(std::move(lv));
}

// Generation k >= 3 on projected vertical lists (proj.cu): the lists of L_{k-1}'s entries from
// those of L_{k-2} (the bitset rows for k = 3), then one popcount-of-AND per candidate over its
// parents' lists.  false: the lists do not fit -- nothing counted, use complete intersection.
// proj_build_begin shared the generation's one host synchronisation with the join
// (the sizes T, sm came back with |C_k|): the list build (pext) on s, overlapping the emitting
// join on the auxiliary stream; the supports wait for both (aux_done).
// The projected lists of L_{k-1} (entry offsets, list build) on the mining stream, right after the
// generation's size read -- before the emitting join is enqueued, so the build starts first.
bool proj_build_stage(gpa_bitset* bs, uint32_t k, DeviceProj& cur, const ProjPending& pp, const uint64_t T[2],
                      const uint32_t sm[4], CountStats* cs) {
  cudaStream_t s = bs->stream;
  GPA_CUDA(cudaEventRecord(cs->e0, s));
  // GPA_PROJ_TEST_MAX_K=k: behave as if the lists of generations > k did not fit (tests drive the
  // mid-run fallback to complete intersection with it)
  const char* tk = getenv("GPA_PROJ_TEST_MAX_K");
  return !(tk && k > (uint32_t)atoi(tk)) && proj_build_finish(pp, T, sm, cur, bs->n_sms, s, cs->ep);
}

// The supports of C_k from the lists (count_proj), once the emitting join (aux stream) is done.
bool proj_count_stage(gpa_bitset* bs, uint32_t k, const DeviceBatch& B, DeviceProj& cur, const ProjPending& pp,
                      bool built, cudaEvent_t aux_done, CountStats* cs, uint64_t src_words) {
  cudaStream_t s = bs->stream;
  const double t0 = now_ms();
  GPA_CUDA(cudaStreamWaitEvent(s, aux_done, 0));
  if (!built) return false;
  bs->d_counts.ensure(B.M, s);
  if (!count_proj_stores_all(cur)) GPA_CUDA(cudaMemsetAsync(bs->d_counts.p, 0, (size_t)B.M * 4, s));
  GPA_CUDA(cudaEventRecord(cs->eb, s));
  cs->build_words = cur.in_words;
  cs->build_bytes = (src_words + cur.words) * 4;            // sources read once, lists written once
  cs->count_bytes = cur.words * 4 + (uint64_t)B.M * 4;      // lists read once, counts written
  launch_count_proj(cur, B.gpar.p, B.ext_off.p, B.eidx.p, B.G, bs->d_counts.p, s);
  cs->kernel = GPA_KERNEL_PROJ;
  cs->launches = 1;
  finish_counts(bs, B.M, cs);
  if (trace_enabled())
    fprintf(stderr, "[gpa] k=%u proj: %u lists, %.1f MB, host %.2f ms\n", k, pp.n, cur.words * 4.0 / 1e6,
            now_ms() - t0);
  return true;
}

// A few page-locked words per thread for the per-generation sizes (one D2H read per generation).
uint32_t* host_sizes() {
  thread_local struct H {
    uint32_t* p = nullptr;
    H() { GPA_CUDA(cudaHostAlloc(reinterpret_cast<void**>(&p), 64, cudaHostAllocDefault)); }
    ~H() { if (p) cudaFreeHost(p); }
  } h;
  return h.p;
}

}  // namespace

// Per thread and device: the level loop's side streams and its events, created once.
struct LoopWs {
  static constexpr int kCopyEvents = 4;
  static constexpr int kEv = 7;   // per generation: [5] start, [0] counting start, [1] counting end,
                                  // [2] all-reduce end, [3, 4) list build, [6] threshold end
  cudaStream_t copy_s = nullptr, aux_s = nullptr;
  cudaEvent_t copy_ev[kCopyEvents] = {}, aux_ev[4] = {}, trace_ev[kEv] = {};
  std::deque<std::array<cudaEvent_t, kEv>> sets;
  explicit LoopWs(int device) {
    use_device(device);
    GPA_CUDA(cudaStreamCreateWithFlags(&copy_s, cudaStreamNonBlocking));
    GPA_CUDA(cudaStreamCreateWithFlags(&aux_s, cudaStreamNonBlocking));
    for (auto& x : copy_ev) GPA_CUDA(cudaEventCreateWithFlags(&x, cudaEventDisableTiming));
    for (auto& x : aux_ev) GPA_CUDA(cudaEventCreateWithFlags(&x, cudaEventDisableTiming));
    for (auto& x : trace_ev) GPA_CUDA(cudaEventCreate(&x));
  }
  cudaEvent_t* evset(size_t i) {
    while (sets.size() <= i) {
      std::array<cudaEvent_t, kEv> a{};
      for (auto& x : a) GPA_CUDA(cudaEventCreate(&x));
      sets.push_back(a);
    }
    return sets[i].data();
  }
  ~LoopWs() {   // at thread exit (errors ignored: the context may be gone)
    for (auto& a : sets)
      for (auto x : a) cudaEventDestroy(x);
    for (auto x : copy_ev) cudaEventDestroy(x);
    for (auto x : aux_ev) cudaEventDestroy(x);
    for (auto x : trace_ev) cudaEventDestroy(x);
    if (copy_s) cudaStreamDestroy(copy_s);
    if (aux_s) cudaStreamDestroy(aux_s);
  }
};
LoopWs& loop_ws(int device) {
  thread_local std::map<int, std::unique_ptr<LoopWs>> m;
  auto& p = m[device];
  if (!p) p = std::make_unique<LoopWs>(device);
  return *p;
}

gpa_result* mine(const gpa_tx_csr* db, uint64_t min_count, const gpa_dist* dist, const gpa_options* opt_in) {
  const double t_start = now_ms();
  NvtxRange nv_mine("gpa_mine");
  HostTrace ht;
  ht.mark("enter", 0);
  gpa_options opt;
  gpa_options_default(&opt);
  if (opt_in) opt = *opt_in;
  GPA_REQUIRE(min_count >= 1, GPA_ERR_INVALID, "min_count must be >= 1");
  const bool keep = (opt.flags & GPA_KEEP_CANDIDATES) != 0;
  const bool fused_requested = opt.count_kernel == GPA_KERNEL_FUSED;
  const bool host_candgen = (opt.flags & GPA_HOST_CANDGEN) != 0;
  const uint32_t max_k = opt.max_k ? opt.max_k : GPA_MAX_K;
  GPA_REQUIRE(min_count < (1ull << 32), GPA_ERR_INVALID, "min_count must be < 2^32");

  bool pairs_ready = false;
  CountStats pair_stats;
  GPA_REQUIRE(db, GPA_ERR_INVALID, "db is NULL");   // a caller bug, not data: checked before any device work
  dist_check(dist);
  use_device(dist ? dist->device : opt.device);
  // the ingest path is chosen collectively: every rank issues the same collective sequence
  const bool overlap = agree_input(db, dist, !(opt.flags & GPA_NO_OVERLAP_INGEST));
  ht.mark("input agreed", 0);
  nvtxRangePushA(overlap ? "gpa_bitset_build (overlapped ingest)" : "gpa_bitset_build");
  gpa_bitset* bs = overlap ? bitset_build_overlapped(db, min_count, dist, &opt, &pairs_ready, &pair_stats)
                           : bitset_build(db, min_count, dist, &opt, true, true);
  struct BsGuard {
    gpa_bitset* b;
    ~BsGuard() { bitset_free(b); }
  } bs_guard{bs};
  nvtxRangePop();
  ht.mark("bitset built", 0);
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

  // ---- the level loop stays on the device: threshold + compaction of the counts into L_k and
  // join + prune of C_{k+1} run as kernels (candgen.cu); only the sizes, the candidate batch (for
  // the trie kernel's host-side plan) and L_k (for the result) cross PCIe.
  DeviceScratch scratch(bs->device);
  DeviceLevel Ld, Ln;   // L_{k-1}, L_k on the device
  DeviceBatch Bd;       // C_k on the device (k >= 3)
  DBuf<uint32_t> d_ior;  // row -> original item id
  // projected vertical lists (GPA_KERNEL_PROJ / AUTO): Pprev = the lists of L_{k-2}'s entries,
  // Pcur = those of L_{k-1} built for generation k (proj.cu)
  DeviceProj* plists = proj_lists(bs->device);
  DeviceProj* Pprev = &plists[0];
  DeviceProj* Pcur = &plists[1];
  if (opt.count_kernel == GPA_KERNEL_FUSED) opt.count_kernel = GPA_KERNEL_AUTO;   // (the multi-kernel fallback)
  bool proj_on = !host_candgen && (opt.count_kernel == GPA_KERNEL_AUTO || opt.count_kernel == GPA_KERNEL_PROJ ||
                                   opt.count_kernel == GPA_KERNEL_PAIRS || opt.count_kernel == GPA_KERNEL_PAIRS_TC) &&
                 bs->pitch_words * 32ull < (1ull << 32);
  if (opt.flags & GPA_COMPLETE_INTERSECTION) proj_on = false;   // the paper's method for k >= 3
  struct Pending {       // a generation's frequent itemsets, still on the device
    size_t level = 0;
    uint32_t F = 0, k = 0;
    bool open = false;                  // |L_k| not yet read back (device-sized level)
    DBuf<uint32_t> items, sup;
  };
  std::vector<Pending> pending;
  // streams and events persist per thread and device (created once: stream and event creation
  // cost ~10 us each, 7 events per generation)
  LoopWs& lw = loop_ws(bs->device);
  struct { cudaStream_t s; } copy_s{lw.copy_s};
  struct SyncAtExit {   // the side streams read `pending` and the level buffers: drained before they go
    cudaStream_t a, b;
    ~SyncAtExit() {
      cudaStreamSynchronize(a);
      cudaStreamSynchronize(b);
    }
  } sync_at_exit{lw.copy_s, lw.aux_s};
  constexpr int kCopyEvents = LoopWs::kCopyEvents;   // re-recorded round robin: a wait captures the event's state at call time
  cudaEvent_t* copy_ev = lw.copy_ev;
  // |L_k| known on the host: record it and start the D2H of L_k (item ids, supports) on the copy
  // stream -- s has just been synchronised, so everything that produced L_k is complete
  auto finalize = [&](Pending& pd, uint32_t F) {
    pd.F = F;
    pd.open = false;
    R->levels[pd.level].n_freq = F;
    R->levels[pd.level].stats.n_freq = F;
    if (F) {
      // one page-locked block of the result: F x k item ids, then F supports
      size_t bytes = (size_t)F * (pd.k + 1) * 4;
      R->pinned.emplace_back(nullptr, 0);
      void* blk = pinned_cache().get(bytes);
      R->pinned.back() = {blk, bytes};
      auto* hi = static_cast<uint32_t*>(blk);
      auto* hs = hi + (size_t)F * pd.k;
      GPA_CUDA(cudaEventRecord(copy_ev[pd.k % kCopyEvents], s));
      GPA_CUDA(cudaStreamWaitEvent(copy_s.s, copy_ev[pd.k % kCopyEvents], 0));
      GPA_CUDA(cudaMemcpyAsync(hi, pd.items.p, (size_t)F * pd.k * 4, cudaMemcpyDeviceToHost, copy_s.s));
      GPA_CUDA(cudaMemcpyAsync(hs, pd.sup.p, (size_t)F * 4, cudaMemcpyDeviceToHost, copy_s.s));
      R->levels[pd.level].fi = hi;
      R->levels[pd.level].fs = hs;
    }
  };
  // a device-sized L_{k-1}: read |L_{k-1}| now (a synchronisation of its own)
  auto settle = [&](DeviceLevel& L) {
    if (!L.n_dev) return;
    uint32_t* hs = host_sizes();
    GPA_CUDA(cudaMemcpyAsync(hs + 15, L.n_dev, 4, cudaMemcpyDeviceToHost, s));
    stream_wait(s);
    L.n = hs[15];
    L.n_dev = nullptr;
    finalize(pending.back(), L.n);
  };
  struct { cudaStream_t s; } aux_s{lw.aux_s};   // the emitting join of C_k, overlapping the list build on s
  struct { cudaEvent_t* e; } aux_evs{lw.aux_ev};  // [0] s -> aux (batch buffers sized), [1] aux done, [2] aux start
  ProjPending ppend;
  bool aux_join = false;     // this generation's batch was emitted on aux_s
  uint64_t pT[2] = {0, 0};
  uint32_t psm[4] = {0, 0, 0, 0};
  // deferred (device-side) timing of a generation on stream s: [5] generation start, [0] counting
  // start, [1] counting end, [2] all-reduce end, [3, 4) projected-list build, [6] threshold end
  struct EvTriple {
    cudaEvent_t* e;           // LoopWs::EvSet::e (kN events)
    bool counted = false;     // e[0..2] recorded (not the generation counted during the overlapped ingest)
  };
  struct EvQueue {            // events[i] uses the workspace's i-th event set
    LoopWs& w;
    std::deque<EvTriple> q;
    EvTriple& emplace_back() { return q.emplace_back(EvTriple{w.evset(q.size())}); }
    void pop_back() { q.pop_back(); }
    EvTriple& operator[](size_t i) { return q[i]; }
    size_t size() const { return q.size(); }
  } events{lw, {}};
  cudaEvent_t* trace_ev = lw.trace_ev;   // GPA_TRACE: [0] end of join stage 1 (s), [1] of the class tables (aux_s)
  std::vector<size_t> event_level;
  d_ior.alloc(std::max<uint32_t>(bs->n_rows, 1), s);
  if (bs->n_rows)
    GPA_CUDA(cudaMemcpyAsync(d_ior.p, bs->item_of_row.data(), bs->n_rows * 4, cudaMemcpyHostToDevice, s));
  uint64_t nL = l1_size(bs);
  if (bs->l1_sub && !bs->l1.empty() && bs->d_l1.n < bs->l1.size()) {   // L_1 -> bitset rows (generation 2)
    bs->d_l1.alloc(bs->l1.size(), s);
    GPA_CUDA(cudaMemcpyAsync(bs->d_l1.p, bs->l1.data(), bs->l1.size() * 4, cudaMemcpyHostToDevice, s));
  }
  // ---- small problems: every generation in one cooperative launch (mine_fused.cu); a capacity
  // overflow falls through to the multi-kernel loop below
  const bool want_fused = !dist && !host_candgen && !(opt.flags & GPA_MULTI_KERNEL) && nL >= 2 &&
                          (fused_requested || opt.count_kernel == GPA_KERNEL_AUTO) &&
                          fused_eligible((uint32_t)nL, bs->pitch_words);
  if (want_fused) {
    FusedOut fo;
    fo.pinned_alloc = [&](size_t& bytes) {   // F lands in a page-locked block of the result
      void* p = pinned_cache().get(bytes);
      R->pinned.emplace_back(p, bytes);
      return p;
    };
    EvTriple& ev = events.emplace_back();
    GPA_CUDA(cudaEventRecord(ev.e[5], s));
    GPA_CUDA(cudaEventRecord(ev.e[0], s));
    // many L_1 rows: generation 2 (a dense contraction) on the tensor cores first, unless the
    // overlapped ingest already counted it
    const uint32_t* c2 = nullptr;
    if (nL > kFusedPairsTcRows) {
      if (!pairs_ready) count_all_pairs(bs, GPA_KERNEL_PAIRS_TC, nullptr);
      c2 = bs->d_counts.p;
    }
    const bool ok = mine_fused(bs->rows.p, bs->pitch_words, bs->n_tx_local, (uint32_t)nL,
                               bs->l1_sub ? bs->d_l1.p : nullptr, d_ior.p, (uint32_t)min_count, max_k, keep,
                               bs->n_sms, s, fo, c2);
    GPA_CUDA(cudaEventRecord(ev.e[1], s));
    GPA_CUDA(cudaEventRecord(ev.e[2], s));
    GPA_CUDA(cudaEventRecord(ev.e[6], s));
    if (ok) {
      ev.counted = true;
      for (const auto& f : fo.levels) {
        gpa_level_data lv;
        lv.k = f.k;
        lv.n_cand = f.M;
        lv.n_freq = f.F;
        lv.n_groups = f.G;
        lv.kept = keep;
        if (f.F) {
          lv.fi = fo.items + f.freq_word;
          lv.fs = fo.sup + f.freq_entry;
        }
        if (keep) {
          lv.cand_items.assign(fo.cand_items.begin() + f.cand_word,
                               fo.cand_items.begin() + f.cand_word + (uint64_t)f.M * f.k);
          lv.cand_counts.assign(fo.cand_counts.begin() + f.cand_entry, fo.cand_counts.begin() + f.cand_entry + f.M);
        }
        lv.stats.n_cand = f.M;
        lv.stats.n_freq = f.F;
        lv.stats.n_groups = f.G;
        lv.stats.kernel = GPA_KERNEL_FUSED;
        lv.stats.launches = R->levels.size() == 1 ? 1 : 0;   // one launch for all generations
        R->levels.push_back(std::move(lv));
      }
      if (R->levels.size() > 1) event_level.push_back(1);   // the whole loop's time on generation 2
      nL = 0;   // skip the multi-kernel loop
    } else {
      events.pop_back();
    }
  }
  ht.mark("loop setup", 0);
  for (uint32_t k = 2; k <= max_k && nL > 0; ++k) {
    double t0 = now_ms();
    char nv_name[32];
    snprintf(nv_name, sizeof nv_name, "gpa_generation %u", k);
    NvtxRange nv_gen(nv_name);
    ht.mark("top", k);
    EvTriple& ev = events.emplace_back();
    GPA_CUDA(cudaEventRecord(ev.e[5], s));
    CountStats cs;
    bool lists_built = false;   // proj_build_stage ran for this generation
    GroupedBatch batch;
    uint64_t M = 0, G = 0;
    if (k == 2) {
      M = nL * (nL - 1) / 2;
      G = nL ? nL - 1 : 0;
    } else if (host_candgen) {
      // reference path (GPA_HOST_CANDGEN): L_{k-1} back to the host, threaded join + prune
      // (runtime/candgen.cpp), the batch up to the device for the device-side threshold
      settle(Ld);
      std::vector<uint32_t> Lh((size_t)Ld.n * (k - 1));
      if (Ld.n) {
        GPA_CUDA(cudaMemcpyAsync(Lh.data(), Ld.rows.p, Lh.size() * 4, cudaMemcpyDeviceToHost, s));
        stream_wait(s);
      }
      batch = candgen_join_prune(Lh, Ld.n, k - 1);
      M = batch.size();
      G = batch.groups();
      GPA_REQUIRE(M < (1ull << 32), GPA_ERR_INVALID, "generation %u has too many candidates", k);
      Bd.k = k;
      Bd.M = (uint32_t)M;
      Bd.G = (uint32_t)G;
      if (M) {
        std::vector<uint32_t> off32(batch.ext_off.begin(), batch.ext_off.end());
        Bd.prefix.ensure(std::max<size_t>(batch.prefix.size(), 1), s);
        Bd.ext_off.ensure(G + 1, s);
        Bd.ext.ensure(M, s);
        GPA_CUDA(cudaMemcpyAsync(Bd.prefix.p, batch.prefix.data(), batch.prefix.size() * 4, cudaMemcpyHostToDevice, s));
        GPA_CUDA(cudaMemcpyAsync(Bd.ext_off.p, off32.data(), (G + 1) * 4, cudaMemcpyHostToDevice, s));
        GPA_CUDA(cudaMemcpyAsync(Bd.ext.p, batch.ext.data(), M * 4, cudaMemcpyHostToDevice, s));
        stream_wait(s);
      }
    } else if (proj_on) {
      aux_join = false;
      // join stage 1 and the projected lists' class tables share one synchronisation; then the
      // emitting join runs on aux_s while the lists are built on s
      const uint32_t* d_sizes = nullptr;
      // the class tables (aux_s) are independent of the join's stage 1 (s): both read L_{k-1}
      // the generation's sizes (|C_k|, groups, list totals, class-table counters, |L_{k-1}|) land in
      // one device block: ONE copy and ONE synchronisation per generation
      uint32_t* blk = scratch.size_block(s);
      const uint32_t n_up = Ld.n_dev ? Ld.n_max : Ld.n;
      // the class scan on s -- a class of L_{k-1} (entries with one left parent) IS a run, so it is
      // the join's run structure too -- then the rest of the class tables on aux beside the join
      const bool lists_ok = proj_build_begin(n_up, Ld.par_a.p, Ld.par_b.p, k == 3 ? nullptr : Pprev, bs->rows.p,
                                             bs->pitch_words, bs->n_rows, scratch, bs->n_sms, aux_s.s, ppend,
                                             Ld.n_dev, blk, s, aux_evs.e[2]);
      if (!lists_ok) proj_on = false;   // lists not addressable: complete intersection from this generation on
      const bool runs = lists_ok && ppend.flag;
      if (device_candgen_begin(Ld, Bd, scratch, bs->n_sms, s, &d_sizes, runs ? ppend.flag : nullptr,
                               runs ? ppend.ex : nullptr, runs ? ppend.bound : nullptr)) {
        if (trace_enabled()) GPA_CUDA(cudaEventRecord(trace_ev[0], s));
        uint32_t* hs = host_sizes();
        if (trace_enabled()) GPA_CUDA(cudaEventRecord(trace_ev[1], aux_s.s));
        GPA_CUDA(cudaEventRecord(aux_evs.e[3], aux_s.s));   // the class tables are done
        GPA_CUDA(cudaStreamWaitEvent(s, aux_evs.e[3], 0));
        GPA_CUDA(cudaMemcpyAsync(hs, blk, 16 * 4, cudaMemcpyDeviceToHost, s));
        // the emitting join (aux) depends on stage 1 only: ordered here, before the list build that
        // s runs right after the read
        GPA_CUDA(cudaEventRecord(aux_evs.e[0], s));
        GPA_CUDA(cudaStreamWaitEvent(aux_s.s, aux_evs.e[0], 0));
        if (trace_enabled()) GPA_CUDA(cudaEventRecord(trace_ev[2], s));
        const double tw0 = now_ms();
        ht.mark("begin enqueued", k);
        stream_wait(s);
        const double tw1 = now_ms();
        ht.mark("sizes back", k);
        if (trace_enabled()) GPA_CUDA(cudaEventRecord(trace_ev[3], s));
        M = hs[0];
        G = hs[1];
        std::memcpy(pT, hs + 2, 16);
        std::memcpy(psm, hs + 6, 16);
        const bool l_open = Ld.n_dev != nullptr;
        if (l_open) {
          Ld.n = hs[10];
          Ld.n_dev = nullptr;
        }
        const double tw2 = now_ms();
        ppend.n = Ld.n;   // the class tables ran over the upper bound; the lists are for |L_{k-1}| entries
        // the list build first (the critical path), then the emitting join on the side stream
        cs.e0 = ev.e[0];
        cs.ep = ev.e[3];
        cs.eb = ev.e[4];
        if (proj_on && M > 0) lists_built = proj_build_stage(bs, k, *Pcur, ppend, pT, psm, &cs);
        device_candgen_finish(Ld, Bd, scratch, bs->n_sms, s, (uint32_t)M, (uint32_t)G, aux_s.s, nullptr);
        GPA_CUDA(cudaEventRecord(aux_evs.e[1], aux_s.s));
        aux_join = true;
        if (l_open) finalize(pending.back(), Ld.n);   // L_{k-1}'s D2H on the copy stream
        ht.mark("join finished", k);
        const double tw3 = now_ms();
        if (trace_enabled()) {
          float ja = 0, jb = 0, jc = 0, jd = 0;
          GPA_CUDA(cudaEventElapsedTime(&ja, ev.e[5], trace_ev[0]));
          GPA_CUDA(cudaEventElapsedTime(&jb, ev.e[5], trace_ev[1]));
          GPA_CUDA(cudaEventElapsedTime(&jc, ev.e[5], trace_ev[2]));
          GPA_CUDA(cudaEventElapsedTime(&jd, ev.e[5], trace_ev[3]));
          fprintf(stderr, "[gpa] k=%u host: enqueue %.3f, wait %.3f, after wait %.3f ms; device: join stage 1 %.3f, "
                  "class tables + sizes %.3f, sizes on s %.3f, host awake %.3f ms (finalize %.3f, finish %.3f)\n", k,
                  tw0 - t0, tw1 - tw0, now_ms() - tw1, ja, jb, jc, jd, tw2 - tw1, tw3 - tw2);
        }
      }
    } else {
      // complete intersection: join + prune on the device, |L_{k-1}| read with the sizes of C_k
      const uint32_t* d_sizes = nullptr;
      if (device_candgen_begin(Ld, Bd, scratch, bs->n_sms, s, &d_sizes)) {
        uint32_t* hs = host_sizes();
        GPA_CUDA(cudaMemcpyAsync(hs, d_sizes, 16 * 4, cudaMemcpyDeviceToHost, s));   // the size block: [10] = |L_{k-1}|
        stream_wait(s);
        if (Ld.n_dev) {
          Ld.n = hs[10];
          Ld.n_dev = nullptr;
          finalize(pending.back(), Ld.n);
        }
        device_candgen_finish(Ld, Bd, scratch, bs->n_sms, s, hs[0], hs[1], s, nullptr);
      }
      M = Bd.M;
      G = Bd.G;
    }
    settle(Ld);   // (candidate generation skipped: fewer than 2 members at most)
    double t1 = now_ms();
    if (M == 0) {
      events.pop_back();
      break;
    }
    cs.e0 = ev.e[0];
    cs.e1 = ev.e[1];
    cs.e2 = ev.e[2];
    cs.ep = ev.e[3];
    cs.eb = ev.e[4];
    GPA_REQUIRE(M < (1ull << 32), GPA_ERR_INVALID, "generation %u has too many candidates", k);
    // the host copy of C_k is needed only for the host-planned kernels and for GPA_KEEP_CANDIDATES
    auto fetch_batch = [&]() {
      if (host_candgen || batch.size() == M) return;
      batch.k = k;
      batch.prefix.resize(G * (k - 1));
      batch.ext.resize(M);
      std::vector<uint32_t> off32(G + 1);
      GPA_CUDA(cudaMemcpyAsync(batch.prefix.data(), Bd.prefix.p, G * (k - 1) * 4, cudaMemcpyDeviceToHost, s));
      GPA_CUDA(cudaMemcpyAsync(off32.data(), Bd.ext_off.p, (G + 1) * 4, cudaMemcpyDeviceToHost, s));
      GPA_CUDA(cudaMemcpyAsync(batch.ext.data(), Bd.ext.p, M * 4, cudaMemcpyDeviceToHost, s));
      stream_wait(s);
      batch.ext_off.assign(off32.begin(), off32.end());
    };
    if (k == 2 && pairs_ready && pairs_kernel_k2(opt.count_kernel)) {
      cs = pair_stats;  // counted during the overlapped ingest
    } else if (k == 2) {
      count_all_pairs(bs, opt.count_kernel, &cs);
    } else {
      const uint64_t src_words = k == 3 ? (uint64_t)bs->n_rows * bs->pitch_words : Pprev->words;
      if (proj_on && proj_count_stage(bs, k, Bd, *Pcur, ppend, lists_built, aux_evs.e[1], &cs, src_words)) {
        std::swap(Pprev, Pcur);
      } else {
        // complete intersection from the static bitset (requested, or the projected lists did not
        // fit: from here on for the remaining generations)
        proj_on = false;
        if (aux_join) GPA_CUDA(cudaStreamWaitEvent(s, aux_evs.e[1], 0));  // the batch came from aux_s
        if (!count_device_batch(bs, Bd, opt.count_kernel, scratch, &cs)) {
          fetch_batch();
          count_grouped(bs, batch, opt.count_kernel, &cs);
        }
      }
    }
    if (keep && k > 2) fetch_batch();
    double t2 = now_ms();
    ht.mark("count enqueued", k);

    // L_k = { c in C_k : count >= min_count } on the device WITHOUT a synchronisation: |L_k| stays on
    // the device (Ln is device-sized) and comes back with the next generation's sizes (or settle())
    // the frequent itemsets of this generation (item ids) and supports for the result, written by
    // the scatter (arrays sized for the upper bound M; the D2H starts once |L_k| is known: finalize)
    Pending pd;
    pd.level = R->levels.size();
    pd.k = k;
    pd.open = true;
    pd.items.alloc((size_t)M * k, s);
    pd.sup.alloc(M, s);
    device_threshold_async(bs->d_counts.p, (uint32_t)M, (uint32_t)min_count, k, l1_size(bs),
                           k == 2 && bs->l1_sub ? bs->d_l1.p : nullptr, Bd.prefix.p, Bd.ext_off.p, Bd.ext.p,
                           (uint32_t)G, host_candgen ? nullptr : Bd.gpar.p, host_candgen ? nullptr : Bd.eidx.p, Ln,
                           scratch, bs->n_sms, s, d_ior.p, pd.items.p, pd.sup.p);
    ev.counted = cs.e0 != nullptr;
    GPA_CUDA(cudaEventRecord(ev.e[6], s));
    std::vector<uint32_t> counts;
    if (keep) {
      counts.resize(M);
      GPA_CUDA(cudaMemcpyAsync(counts.data(), bs->d_counts.p, M * 4, cudaMemcpyDeviceToHost, s));
      stream_wait(s);
    }
    const double tr0 = now_ms();
    ht.mark("threshold enqueued", k);
    record_level(R, bs, k, k > 2 ? &batch : nullptr, M, {}, {}, keep, keep ? &counts : nullptr);
    R->levels.back().n_freq = 0;   // set by finalize()
    pending.push_back(std::move(pd));
    std::swap(Ld, Ln);
    nL = M;   // an upper bound of |L_k|: the next generation's candidate count decides
    if (trace_enabled())
      fprintf(stderr, "[gpa] k=%u M=%llu G=%llu: candgen %.2f ms, count phase %.2f ms, threshold enqueue %.2f ms "
              "(record %.2f)\n", k, (unsigned long long)M, (unsigned long long)G, t1 - t0, t2 - t1, now_ms() - t2,
              now_ms() - tr0);
    event_level.push_back(R->levels.size() - 1);
    gpa_level_stats& st = R->levels.back().stats;
    st.n_cand = M;
    st.n_groups = G;
    st.kernel = cs.kernel;
    st.launches = cs.launches;
    st.count_ms = cs.count_ms;
    st.allreduce_ms = cs.allreduce_ms;
    st.candgen_ms = t1 - t0;
    st.build_words = cs.build_words;
    st.build_bytes = cs.build_bytes;
    st.count_bytes = cs.count_bytes;
  }

  settle(Ld);   // the last generation's |L_k| (when the loop ended on max_k)
  // ---- deferred: kernel times and the frequent itemsets of every generation
  const double tf0 = now_ms();
  stream_wait(s);
  stream_wait(copy_s.s);
  ht.mark("drained", 0);
  const double tf1 = now_ms();
  // phases of the level loop from the events on s (device time, contiguous per generation):
  // candidate generation = generation start -> counting start, counting (+ all-reduce) = counting
  // start -> all-reduce end, threshold = all-reduce end -> threshold end
  for (size_t i = 0; i < event_level.size(); ++i) {
    const EvTriple& E = events[i];
    gpa_level_stats& st = R->levels[event_level[i]].stats;
    float g = 0;
    GPA_CUDA(cudaEventElapsedTime(&g, E.e[5], E.e[6]));
    if (!E.counted) {   // generation 2 counted during the overlapped ingest: stats from the ingest
      R->phase_ms[GPA_PHASE_THRESHOLD] += g;
      continue;
    }
    float a = 0, b = 0, cg = 0;
    GPA_CUDA(cudaEventElapsedTime(&a, E.e[0], E.e[1]));
    GPA_CUDA(cudaEventElapsedTime(&b, E.e[1], E.e[2]));
    GPA_CUDA(cudaEventElapsedTime(&cg, E.e[5], E.e[0]));
    if (st.kernel == GPA_KERNEL_PROJ) {
      float c = 0;
      GPA_CUDA(cudaEventElapsedTime(&c, E.e[3], E.e[4]));
      st.build_ms = c;
      GPA_CUDA(cudaEventElapsedTime(&c, E.e[0], E.e[3]));
      st.setup_ms = c;
    }
    st.count_ms = a;
    st.allreduce_ms = dist ? b : 0.0;
    if (trace_enabled()) {   // device timeline of the generation (ms from the previous one's end)
      float gap = 0;
      if (i > 0) GPA_CUDA(cudaEventElapsedTime(&gap, events[i - 1].e[6], E.e[5]));
      fprintf(stderr, "[gpa] gen %u: gap %.3f candgen %.3f setup %.3f build %.3f count %.3f threshold %.3f\n",
              R->levels[event_level[i]].k, gap, cg, st.kernel == GPA_KERNEL_PROJ ? st.setup_ms : 0.0,
              st.kernel == GPA_KERNEL_PROJ ? st.build_ms : 0.0, a, g - cg - a - b);
    }
    R->phase_ms[GPA_PHASE_CANDGEN] += cg;
    R->phase_ms[GPA_PHASE_COUNT] += a + b;
    R->phase_ms[GPA_PHASE_THRESHOLD] += g - cg - a - b;
  }
  // F is already in the result's page-locked blocks (copy stream drained above)
  pending.clear();
  ht.mark("F in the result", 0);
  if (trace_enabled())
    fprintf(stderr, "[gpa] end of loop: drain %.2f ms, F transfer %.2f ms\n", tf1 - tf0, now_ms() - tf1);

  uint64_t acc = 0;
  for (auto& lv : R->levels) {
    R->freq_start.push_back(acc);
    acc += lv.n_freq;
  }
  R->freq_start.push_back(acc);
  R->phase_ms[GPA_PHASE_TOTAL] = now_ms() - t_start;
  ht.mark("return", 0);
  ht.print();
  r_guard.r = nullptr;
  return R;
}

}  // namespace gpa

// ---------------------------------------------------------------- C ABI: mine + result

extern "C" gpa_status gpa_mine(const gpa_tx_csr* db, uint64_t min_count, const gpa_dist* dist, const gpa_options* opt,
                               gpa_result** out) {
  return gpa::guard([&] {
    GPA_REQUIRE(out, GPA_ERR_INVALID, "out is NULL");
    gpa::DistScope scope(dist);
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
    if (items) *items = lv.items() + j * lv.k;
    if (k) *k = lv.k;
    if (support) *support = lv.supports()[j];
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
    if (items) *items = lv.items();
    if (supports) *supports = lv.supports();
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

extern "C" uint64_t gpa_kernel_launches(void) { return gpa::g_kernel_launches.load(std::memory_order_relaxed); }
