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
#include <cstdlib>
#include <cstring>
#include <deque>

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

struct gpa_level_data {
  uint32_t k = 0;
  uint64_t n_cand = 0, n_freq = 0, n_groups = 0;
  FVec freq_items;                     // n_freq * k, original ids, lexicographic
  FVec freq_support;                   // n_freq
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
bool count_projected_staged(gpa_bitset* bs, uint32_t k, const DeviceBatch& B, DeviceProj& cur, const ProjPending& pp,
                            const uint64_t T[2], const uint32_t sm[4], cudaEvent_t aux_done, CountStats* cs,
                            uint64_t src_words) {
  cudaStream_t s = bs->stream;
  const double t0 = now_ms();
  GPA_CUDA(cudaEventRecord(cs->e0, s));
  // GPA_PROJ_TEST_MAX_K=k: behave as if the lists of generations > k did not fit (tests drive the
  // mid-run fallback to complete intersection with it)
  const char* tk = getenv("GPA_PROJ_TEST_MAX_K");
  const bool ok = !(tk && k > (uint32_t)atoi(tk)) && proj_build_finish(pp, T, sm, cur, bs->n_sms, s, cs->ep);
  GPA_CUDA(cudaStreamWaitEvent(s, aux_done, 0));
  if (!ok) return false;
  bs->d_counts.ensure(B.M, s);
  GPA_CUDA(cudaMemsetAsync(bs->d_counts.p, 0, (size_t)B.M * 4, s));
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

// Page-locked staging for the frequent itemsets: each generation's L_k (item ids, supports) is
// copied to the host right after its threshold, overlapping the next generations, into blocks
// that persist per thread across calls (grow-only); the result vectors are filled from them at
// the end (a pageable D2H of all of F took ~3 ms at the end of the loop on T40I10D10M).
struct PinnedArena {
  std::vector<std::pair<uint8_t*, size_t>> blocks;
  size_t cur = 0, used = 0;
  void reset() { cur = 0; used = 0; }
  void* get(size_t bytes) {
    bytes = (bytes + 255) & ~size_t(255);
    while (cur < blocks.size() && used + bytes > blocks[cur].second) {
      ++cur;
      used = 0;
    }
    if (cur == blocks.size()) {
      const size_t sz = std::max<size_t>(bytes, size_t(64) << 20);
      void* p = nullptr;
      GPA_CUDA(cudaHostAlloc(&p, sz, cudaHostAllocDefault));
      blocks.emplace_back(static_cast<uint8_t*>(p), sz);
      used = 0;
    }
    void* r = blocks[cur].first + used;
    used += bytes;
    return r;
  }
  ~PinnedArena() {
    for (auto& b : blocks) cudaFreeHost(b.first);
  }
};

PinnedArena& pinned_arena() {
  thread_local PinnedArena a;
  return a;
}

}  // namespace

gpa_result* mine(const gpa_tx_csr* db, uint64_t min_count, const gpa_dist* dist, const gpa_options* opt_in) {
  const double t_start = now_ms();
  gpa_options opt;
  gpa_options_default(&opt);
  if (opt_in) opt = *opt_in;
  GPA_REQUIRE(min_count >= 1, GPA_ERR_INVALID, "min_count must be >= 1");
  const bool keep = (opt.flags & GPA_KEEP_CANDIDATES) != 0;
  const bool fused_requested = opt.count_kernel == GPA_KERNEL_FUSED;
  pinned_arena().reset();  // a previous call on this thread consumed its blocks before returning
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
  gpa_bitset* bs = overlap ? bitset_build_overlapped(db, min_count, dist, &opt, &pairs_ready, &pair_stats)
                           : bitset_build(db, min_count, dist, &opt, true, true);
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

  // ---- the level loop stays on the device: threshold + compaction of the counts into L_k and
  // join + prune of C_{k+1} run as kernels (candgen.cu); only the sizes, the candidate batch (for
  // the trie kernel's host-side plan) and L_k (for the result) cross PCIe.
  DeviceScratch scratch;
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
    const uint32_t* h_items = nullptr;  // page-locked copies (pinned_arena)
    const uint32_t* h_sup = nullptr;
  };
  std::vector<Pending> pending;
  struct CopyStream {
    cudaStream_t s = nullptr;
    CopyStream() { GPA_CUDA(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking)); }
    ~CopyStream() {
      if (s) { cudaStreamSynchronize(s); cudaStreamDestroy(s); }
    }
  } copy_s;
  constexpr int kCopyEvents = 4;   // re-recorded round robin: a wait captures the event's state at call time
  struct Events {
    cudaEvent_t e[kCopyEvents] = {};
    Events() { for (auto& x : e) GPA_CUDA(cudaEventCreateWithFlags(&x, cudaEventDisableTiming)); }
    ~Events() { for (auto x : e) if (x) cudaEventDestroy(x); }
  } copy_evs;
  cudaEvent_t* copy_ev = copy_evs.e;
  // |L_k| known on the host: record it and start the D2H of L_k (item ids, supports) on the copy
  // stream -- s has just been synchronised, so everything that produced L_k is complete
  auto finalize = [&](Pending& pd, uint32_t F) {
    pd.F = F;
    pd.open = false;
    R->levels[pd.level].n_freq = F;
    R->levels[pd.level].stats.n_freq = F;
    if (F) {
      auto* hi = static_cast<uint32_t*>(pinned_arena().get((size_t)F * pd.k * 4));
      auto* hs = static_cast<uint32_t*>(pinned_arena().get((size_t)F * 4));
      GPA_CUDA(cudaEventRecord(copy_ev[pd.k % kCopyEvents], s));
      GPA_CUDA(cudaStreamWaitEvent(copy_s.s, copy_ev[pd.k % kCopyEvents], 0));
      GPA_CUDA(cudaMemcpyAsync(hi, pd.items.p, (size_t)F * pd.k * 4, cudaMemcpyDeviceToHost, copy_s.s));
      GPA_CUDA(cudaMemcpyAsync(hs, pd.sup.p, (size_t)F * 4, cudaMemcpyDeviceToHost, copy_s.s));
      pd.h_items = hi;
      pd.h_sup = hs;
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
  CopyStream aux_s;          // the emitting join of C_k, overlapping the list build on s
  Events aux_evs;            // [0] s -> aux (batch buffers sized), [1] aux done
  ProjPending ppend;
  bool aux_join = false;     // this generation's batch was emitted on aux_s
  uint64_t pT[2] = {0, 0};
  uint32_t psm[4] = {0, 0, 0, 0};
  // deferred (device-side) timing of a generation on stream s: [5] generation start, [0] counting
  // start, [1] counting end, [2] all-reduce end, [3, 4) projected-list build, [6] threshold end
  struct EvTriple {
    enum { kN = 7 };
    cudaEvent_t e[kN] = {};
    bool counted = false;   // e[0..2] recorded (not the generation counted during the overlapped ingest)
    EvTriple() {
      for (auto& x : e) GPA_CUDA(cudaEventCreate(&x));
    }
    EvTriple(EvTriple&& o) noexcept {
      for (int i = 0; i < kN; ++i) std::swap(e[i], o.e[i]);
      counted = o.counted;
    }
    EvTriple(const EvTriple&) = delete;
    ~EvTriple() {
      for (auto x : e)
        if (x) cudaEventDestroy(x);
    }
  };
  std::deque<EvTriple> events;
  EvTriple trace_evs;        // GPA_TRACE: [0] end of join stage 1 (s), [1] of the class tables (aux_s)
  cudaEvent_t* trace_ev = trace_evs.e;
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
        lv.freq_items.assign(fo.items.begin() + f.freq_word, fo.items.begin() + f.freq_word + (uint64_t)f.F * f.k);
        lv.freq_support.assign(fo.sup.begin() + f.freq_entry, fo.sup.begin() + f.freq_entry + f.F);
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
  for (uint32_t k = 2; k <= max_k && nL > 0; ++k) {
    double t0 = now_ms();
    EvTriple& ev = events.emplace_back();
    GPA_CUDA(cudaEventRecord(ev.e[5], s));
    CountStats cs;
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
      GPA_CUDA(cudaEventRecord(aux_evs.e[2], s));
      GPA_CUDA(cudaStreamWaitEvent(aux_s.s, aux_evs.e[2], 0));
      // L_{k-1} is device-sized: |L_{k-1}| comes back with the sizes of C_k and of the lists -- ONE
      // synchronisation per generation
      const uint32_t n_up = Ld.n_dev ? Ld.n_max : Ld.n;
      if (device_candgen_begin(Ld, Bd, scratch, bs->n_sms, s, &d_sizes)) {
        if (trace_enabled()) GPA_CUDA(cudaEventRecord(trace_ev[0], s));
        uint32_t* hs = host_sizes();
        if (proj_build_begin(n_up, Ld.par_a.p, Ld.par_b.p, k == 3 ? nullptr : Pprev, bs->rows.p, bs->pitch_words,
                             bs->n_rows, scratch, bs->n_sms, aux_s.s, ppend, Ld.n_dev)) {
          GPA_CUDA(cudaMemcpyAsync(hs + 2, ppend.d_tot, 16, cudaMemcpyDeviceToHost, aux_s.s));
          GPA_CUDA(cudaMemcpyAsync(hs + 6, ppend.d_small, 16, cudaMemcpyDeviceToHost, aux_s.s));
        } else {
          proj_on = false;   // lists not addressable: complete intersection from this generation on
        }
        if (trace_enabled()) GPA_CUDA(cudaEventRecord(trace_ev[1], aux_s.s));
        GPA_CUDA(cudaMemcpyAsync(hs, d_sizes, 8, cudaMemcpyDeviceToHost, s));
        if (Ld.n_dev) GPA_CUDA(cudaMemcpyAsync(hs + 10, Ld.n_dev, 4, cudaMemcpyDeviceToHost, s));
        if (trace_enabled()) GPA_CUDA(cudaEventRecord(trace_ev[2], s));
        const double tw0 = now_ms();
        stream_wait(s);
        stream_wait(aux_s.s);
        const double tw1 = now_ms();
        if (trace_enabled()) GPA_CUDA(cudaEventRecord(trace_ev[3], s));
        M = hs[0];
        G = hs[1];
        std::memcpy(pT, hs + 2, 16);
        std::memcpy(psm, hs + 6, 16);
        if (Ld.n_dev) {
          Ld.n = hs[10];
          Ld.n_dev = nullptr;
          finalize(pending.back(), Ld.n);
        }
        const double tw2 = now_ms();
        ppend.n = Ld.n;   // the class tables ran over the upper bound; the lists are for |L_{k-1}| entries
        device_candgen_finish(Ld, Bd, scratch, bs->n_sms, s, (uint32_t)M, (uint32_t)G, aux_s.s, aux_evs.e[0]);
        GPA_CUDA(cudaEventRecord(aux_evs.e[1], aux_s.s));
        aux_join = true;
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
        GPA_CUDA(cudaMemcpyAsync(hs, d_sizes, 8, cudaMemcpyDeviceToHost, s));
        if (Ld.n_dev) GPA_CUDA(cudaMemcpyAsync(hs + 10, Ld.n_dev, 4, cudaMemcpyDeviceToHost, s));
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
      if (proj_on && count_projected_staged(bs, k, Bd, *Pcur, ppend, pT, psm, aux_evs.e[1], &cs, src_words)) {
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

    // L_k = { c in C_k : count >= min_count } on the device WITHOUT a synchronisation: |L_k| stays on
    // the device (Ln is device-sized) and comes back with the next generation's sizes (or settle())
    device_threshold_async(bs->d_counts.p, (uint32_t)M, (uint32_t)min_count, k, l1_size(bs),
                           k == 2 && bs->l1_sub ? bs->d_l1.p : nullptr, Bd.prefix.p, Bd.ext_off.p, Bd.ext.p,
                           (uint32_t)G, host_candgen ? nullptr : Bd.gpar.p, host_candgen ? nullptr : Bd.eidx.p, Ln,
                           scratch, bs->n_sms, s);
    // the frequent itemsets of this generation (item ids) and supports, mapped on the device (over
    // the upper bound M; the kernel stops at |L_k|); their D2H starts once |L_k| is known (finalize)
    Pending pd;
    pd.level = R->levels.size();
    pd.k = k;
    pd.open = true;
    pd.items.alloc((size_t)M * k, s);
    pd.sup.alloc(M, s);
    device_map_items(Ln.rows.p, (uint64_t)M * k, d_ior.p, pd.items.p, bs->n_sms, s, Ln.n_dev, k, Ln.sup.p, pd.sup.p);
    ev.counted = cs.e0 != nullptr;
    GPA_CUDA(cudaEventRecord(ev.e[6], s));
    std::vector<uint32_t> counts;
    if (keep) {
      counts.resize(M);
      GPA_CUDA(cudaMemcpyAsync(counts.data(), bs->d_counts.p, M * 4, cudaMemcpyDeviceToHost, s));
      stream_wait(s);
    }
    const double tr0 = now_ms();
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
  // pinned staging -> the result's vectors: sized first, then copied in ~256 KB pieces over the pool
  // (one generation can hold most of F)
  struct Piece { size_t i; uint64_t a, b; };
  std::vector<Piece> pieces;
  for (size_t i = 0; i < pending.size(); ++i) {
    const Pending& pd = pending[i];
    gpa_level_data& lv = R->levels[pd.level];
    lv.freq_items.resize((size_t)pd.F * pd.k);
    lv.freq_support.resize(pd.F);
    const uint64_t step = std::max<uint64_t>(1, (uint64_t)65536 / std::max<uint32_t>(pd.k, 1));
    for (uint64_t a = 0; a < pd.F; a += step) pieces.push_back({i, a, std::min<uint64_t>(pd.F, a + step)});
  }
  parallel_for(pieces.size(), [&](size_t j) {
    const Piece& pc = pieces[j];
    const Pending& pd = pending[pc.i];
    gpa_level_data& lv = R->levels[pd.level];
    std::memcpy(lv.freq_items.data() + pc.a * pd.k, pd.h_items + pc.a * pd.k, (pc.b - pc.a) * pd.k * 4);
    std::memcpy(lv.freq_support.data() + pc.a, pd.h_sup + pc.a, (pc.b - pc.a) * 4);
  });
  pending.clear();
  if (trace_enabled())
    fprintf(stderr, "[gpa] end of loop: drain %.2f ms, F transfer %.2f ms\n", tf1 - tf0, now_ms() - tf1);

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

extern "C" uint64_t gpa_kernel_launches(void) { return gpa::g_kernel_launches.load(std::memory_order_relaxed); }
