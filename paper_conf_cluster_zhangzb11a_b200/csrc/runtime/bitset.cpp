// Static bitset construction and the counting engine (host side of the library).
//
// gpa_bitset_create / gpa_mine share bitset_build():
//   upload (host CSR only) -> device validation + generation-1 histogram (P13@338)
//   -> all-reduce of the histogram across ranks -> rows = items with count >= row_min_count,
//   ascending item id -> device transpose of the CSR into the static bitset (P18@755).
// count_grouped / count_all_pairs run the sm_100a counting kernels on a candidate batch and
// leave the (rank-summed) counts in bs->d_counts.
#include <cstring>
#include <algorithm>
#include <chrono>
#include <cstdlib>
#include <numeric>

#include "internal.h"

namespace gpa {

// AUTO's choice between the streaming prefix kernel (mean sibling group >= cut) and the trie walk
// (cut 8: T40I10D10M generation 3, 4.6 siblings per group, runs 6.3 ms as a trie walk vs 7.0 ms streamed);
// GPA_AUTO_SIBLINGS overrides the cut (experiments only)
static double auto_sibling_cut() {
  static const double cut = [] {
    const char* e = getenv("GPA_AUTO_SIBLINGS");
    return e ? atof(e) : 8.0;
  }();
  return cut;
}

namespace {

void launch_trie(uint32_t k, const uint32_t* rows, uint64_t pitch_words, const TrieBlock* blocks,
                 const uint32_t* block_rows, const uint4* lrows, const uint8_t* lcp, uint32_t n_blocks,
                 uint32_t max_rows, uint32_t n_parts, uint32_t* counts, cudaStream_t s) {
  launch_count_trie(k, rows, pitch_words, blocks, block_rows, lrows, lcp, n_blocks, max_rows, n_parts, counts, s);
}

double now_ms() {
  return std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now().time_since_epoch()).count();
}

float event_ms(cudaEvent_t a, cudaEvent_t b) {
  float ms = 0;
  GPA_CUDA(cudaEventElapsedTime(&ms, a, b));
  return ms;
}

void validate_options(const gpa_options& o) {
  GPA_REQUIRE(o.count_kernel <= GPA_KERNEL_FUSED, GPA_ERR_INVALID, "unknown count_kernel %u", o.count_kernel);
  GPA_REQUIRE(o.max_k <= GPA_MAX_K, GPA_ERR_INVALID, "max_k %u > GPA_MAX_K", o.max_k);
  GPA_REQUIRE(!o.reserved[0] && !o.reserved[1] && !o.reserved[2], GPA_ERR_INVALID, "reserved option fields must be 0");
  GPA_REQUIRE((o.flags & ~(GPA_KEEP_CANDIDATES | GPA_HOST_CANDGEN | GPA_NO_OVERLAP_INGEST | GPA_COMPLETE_INTERSECTION |
                           GPA_MULTI_KERNEL)) == 0,
              GPA_ERR_INVALID, "unknown option flags 0x%x", o.flags);
}

}  // namespace

gpa_bitset* bitset_build(const gpa_tx_csr* db, uint64_t row_min_count, const gpa_dist* dist, const gpa_options* opt_in,
                         bool prechecked, bool keep_all_rows) {
  GPA_REQUIRE(db, GPA_ERR_INVALID, "db is NULL");   // a caller bug, not data: checked before any device work
  gpa_options opt;
  gpa_options_default(&opt);
  if (opt_in) opt = *opt_in;
  validate_options(opt);
  dist_check(dist);
  DeviceInfo di = use_device(dist ? dist->device : opt.device);
  if (!prechecked) agree_input(db, dist, false);

  auto* bs = new gpa_bitset();
  struct Guard {
    gpa_bitset* b;
    ~Guard() { if (b) bitset_free(b); }
  } guard{bs};
  bs->device = di.device;
  bs->n_sms = di.n_sms;
  bs->dist = dist;
  bs->opt = opt;
  bs->n_items = db->n_items;
  bs->n_tx_local = db->n_tx;
  bs->bundle = acquire_bundle(bs->device);
  bs->stream = opt.stream ? static_cast<cudaStream_t>(opt.stream) : bs->bundle->s;
  bs->ev0 = bs->bundle->ev[0];
  bs->ev1 = bs->bundle->ev[1];
  bs->ev2 = bs->bundle->ev[2];
  cudaStream_t s = bs->stream;

  // ---- input on the device
  double t0 = now_ms();
  const uint64_t n_tx = db->n_tx;
  uint64_t nnz = 0;
  DBuf<uint64_t> d_off;
  DBuf<uint32_t> d_items;
  const uint64_t* off_dev = db->offsets;
  const uint32_t* items_dev = db->items;
  uint64_t first_off = 0;
  if (db->memory == GPA_MEM_HOST) {
    if (n_tx) {
      first_off = db->offsets[0];
      nnz = db->offsets[n_tx];
    }
    GPA_REQUIRE(first_off == 0, GPA_ERR_INVALID, "offsets[0] must be 0");
    GPA_REQUIRE(db->items || nnz == 0, GPA_ERR_INVALID, "db->items is NULL");
    d_off.alloc(n_tx + 1, s);
    GPA_CUDA(cudaMemcpyAsync(d_off.p, db->offsets, (n_tx + 1) * sizeof(uint64_t), cudaMemcpyHostToDevice, s));
    if (nnz) {
      d_items.alloc(nnz, s);
      GPA_CUDA(cudaMemcpyAsync(d_items.p, db->items, nnz * sizeof(uint32_t), cudaMemcpyHostToDevice, s));
    }
    off_dev = d_off.p;
    items_dev = d_items.p;
  } else if (n_tx) {
    GPA_CUDA(cudaMemcpyAsync(&first_off, db->offsets, sizeof(uint64_t), cudaMemcpyDeviceToHost, s));
    GPA_CUDA(cudaMemcpyAsync(&nnz, db->offsets + n_tx, sizeof(uint64_t), cudaMemcpyDeviceToHost, s));
    stream_wait(s);
    GPA_REQUIRE(first_off == 0, GPA_ERR_INVALID, "offsets[0] must be 0");
  }
  stream_wait(s);
  double t1 = now_ms();
  bs->build_ms[0] = t1 - t0;

  // ---- validation + generation-1 histogram (+ n_tx) ; one all-reduce each
  const uint32_t n_items = db->n_items;
  // one block: the histogram (n_items words, rounded to even), the flags word + pad, n_tx (u64):
  // one memset, one H2D of n_tx, one D2H of everything after the collectives
  const size_t nh = (std::max<uint32_t>(n_items, 1) + 1) & ~size_t(1);
  DBuf<uint32_t> d_blk;
  d_blk.alloc(nh + 4, s);
  uint32_t* const d_hist_p = d_blk.p;
  uint32_t* const d_flags_p = d_blk.p + nh;
  uint64_t* const d_ntx_p = reinterpret_cast<uint64_t*>(d_blk.p + nh + 2);
  GPA_CUDA(cudaMemsetAsync(d_blk.p, 0, (nh + 2) * sizeof(uint32_t), s));
  GPA_CUDA(cudaMemcpyAsync(d_ntx_p, &bs->n_tx_local, sizeof(uint64_t), cudaMemcpyHostToDevice, s));
  struct { uint32_t* p; } d_hist{d_hist_p}, d_flags{d_flags_p};
  struct { uint64_t* p; } d_ntx{d_ntx_p};
  bs->pitch_words = pitch_words_for(n_tx);
  // up to 1,024 item ids: ONE read of the CSR builds the rows of every item id and their popcounts
  // are the generation-1 counts (scan_build); the L_1 rows are compacted afterwards.  Otherwise a
  // histogram pass, then the build of the L_1 rows (a second read).
  const bool scan = n_tx > 0 && scan_build_supported(n_items, items_dev);
  uint32_t flags = 0;
  if (scan) {
    bs->rows.alloc((size_t)n_items * bs->pitch_words, s);
    launch_scan_build(off_dev, items_dev, n_tx, nnz, n_items, bs->pitch_words, bs->rows.p, d_hist.p, d_flags.p, s);
  } else {
    launch_hist_validate(off_dev, items_dev, n_tx, nnz, n_items, d_hist.p, d_flags.p, bs->n_sms, s);
    GPA_CUDA(cudaMemcpyAsync(&flags, d_flags.p, sizeof(uint32_t), cudaMemcpyDeviceToHost, s));
    stream_wait(s);
    if ((flags & kFlagNonCanonical) && !(flags & (kFlagBadItem | kFlagBadOffsets))) {
      GPA_CUDA(cudaMemsetAsync(d_hist.p, 0, n_items * sizeof(uint32_t), s));
      launch_hist_dedup(off_dev, items_dev, n_tx, nnz, n_items, d_hist.p, bs->n_sms, s);
    }
  }
  allreduce_max_u32(dist, d_flags.p, 1, s);   // every rank takes the same accept / reject decision
  allreduce_sum_u32(dist, d_hist.p, n_items, s);
  allreduce_sum_u64(dist, d_ntx.p, 1, s);
  std::vector<uint32_t> h_blk(nh + 4);
  GPA_CUDA(cudaMemcpyAsync(h_blk.data(), d_blk.p, (nh + 4) * sizeof(uint32_t), cudaMemcpyDeviceToHost, s));
  stream_wait(s);
  bs->item_counts.assign(h_blk.begin(), h_blk.begin() + n_items);
  flags = h_blk[nh];
  std::memcpy(&bs->n_tx_global, h_blk.data() + nh + 2, sizeof(uint64_t));
  GPA_REQUIRE(!(flags & kFlagBadOffsets), GPA_ERR_INVALID, "offsets are not non-decreasing%s",
              dist ? " (on some rank)" : "");
  GPA_REQUIRE(!(flags & kFlagBadItem), GPA_ERR_INVALID, "an item id is >= n_items (%u)%s", n_items,
              dist ? " (on some rank)" : "");
  GPA_REQUIRE(bs->n_tx_global < (1ull << 32), GPA_ERR_INVALID, "n_tx must be < 2^32 (32-bit supports)");
  double t2 = now_ms();
  bs->build_ms[1] = t2 - t1;

  // ---- rows: items with count >= row_min_count, ascending id (Q8, Q14); row_min_count
  // 0: every item id owns a row, absent items an all-zero one (shards of one database then share
  // one row set without a collective)
  bs->row_of_item.assign(n_items, -1);
  for (uint32_t i = 0; i < n_items; ++i) {
    if (row_min_count == 0 || (bs->item_counts[i] >= row_min_count && bs->item_counts[i] > 0)) {
      bs->row_of_item[i] = (int32_t)bs->item_of_row.size();
      bs->item_of_row.push_back(i);
    }
  }
  bs->n_rows = (uint32_t)bs->item_of_row.size();
  if (scan && keep_all_rows) {
    // the one-pass build left a row for every item id: keep them (row = item id) and list L_1
    bs->l1 = bs->item_of_row;
    bs->item_of_row.resize(n_items);
    for (uint32_t i = 0; i < n_items; ++i) {
      bs->item_of_row[i] = i;
      bs->row_of_item[i] = (int32_t)i;
    }
    bs->n_rows = n_items;
    bs->l1_sub = bs->l1.size() < n_items;   // else every row is in L_1
  } else if (scan) {
    // row r <- row item_of_row[r] from the first row whose item differs (in place)
    uint32_t r0 = 0;
    while (r0 < bs->n_rows && bs->item_of_row[r0] == r0) ++r0;
    if (r0 < bs->n_rows) {
      DBuf<uint32_t> d_sel;
      d_sel.alloc(bs->n_rows, s);
      GPA_CUDA(cudaMemcpyAsync(d_sel.p, bs->item_of_row.data(), bs->n_rows * sizeof(uint32_t), cudaMemcpyHostToDevice,
                               s));
      launch_compact_rows(bs->rows.p, d_sel.p, r0, bs->n_rows, bs->pitch_words, bs->n_sms, s);
      stream_wait(s);   // d_sel is freed at scope exit (stream-ordered, but keep the phase timing honest)
    }
  } else if (bs->n_rows) {
    DBuf<int32_t> d_map;
    d_map.alloc(n_items, s);
    GPA_CUDA(cudaMemcpyAsync(d_map.p, bs->row_of_item.data(), n_items * sizeof(int32_t), cudaMemcpyHostToDevice, s));
    bs->rows.alloc((size_t)bs->n_rows * bs->pitch_words, s);
    launch_bitset_build(off_dev, items_dev, n_tx, nnz, d_map.p, n_items, bs->n_rows, bs->pitch_words, bs->rows.p, 0,
                        n_tx, s);
  }
  stream_wait(s);
  bs->build_ms[2] = now_ms() - t2;
  guard.b = nullptr;
  return bs;
}

void bitset_free(gpa_bitset* bs) {
  if (!bs) return;
  if (bs->stream) cudaStreamSynchronize(bs->stream);
  bs->rows.reset();
  bs->d_counts.reset();
  bs->d_prefix.reset();
  bs->d_ext.reset();
  bs->d_flat.reset();
  bs->d_tasks.reset();
  bs->d_tblocks.reset();
  bs->d_trows.reset();
  bs->d_lrows.reset();
  bs->d_lcp.reset();
  bs->d_cgroup.reset();
  bs->d_l1.reset();
  bs->d_pairs_all.reset();
  if (bs->stream) cudaStreamSynchronize(bs->stream);
  if (bs->bundle) {
    cudaStreamSynchronize(bs->bundle->s);
    release_bundle(bs->bundle);   // its stream is idle: reusable by the next bitset
  }
  delete bs;
}

// ------------------------------------------------------------------ counting engine

namespace {

// start / end events of a counting launch: the caller's (deferred timing, no sync) or the bitset's
cudaEvent_t ev_start(gpa_bitset* bs, CountStats* st) { return st && st->e0 ? st->e0 : bs->ev0; }

}  // namespace

void finish_counts(gpa_bitset* bs, size_t M, CountStats* st) {
  cudaStream_t s = bs->stream;
  const bool deferred = st && st->e0;
  cudaEvent_t e1 = deferred ? st->e1 : bs->ev1, e2 = deferred ? st->e2 : bs->ev2;
  GPA_CUDA(cudaEventRecord(e1, s));
  allreduce_sum_u32(bs->dist, bs->d_counts.p, M, s);
  GPA_CUDA(cudaEventRecord(e2, s));
  if (deferred) return;
  GPA_CUDA(cudaEventSynchronize(e2));
  if (st) {
    st->count_ms = event_ms(bs->ev0, bs->ev1);
    st->allreduce_ms = bs->dist ? event_ms(bs->ev1, bs->ev2) : 0.0;
  }
}

namespace {

void count_flat_v0(gpa_bitset* bs, const std::vector<uint32_t>& flat, uint32_t k, uint64_t M, CountStats* st) {
  cudaStream_t s = bs->stream;
  bs->d_flat.ensure(std::max<size_t>(flat.size(), 1), s);
  bs->d_counts.ensure(std::max<uint64_t>(M, 1), s);
  GPA_CUDA(cudaMemcpyAsync(bs->d_flat.p, flat.data(), flat.size() * sizeof(uint32_t), cudaMemcpyHostToDevice, s));
  GPA_CUDA(cudaEventRecord(ev_start(bs, st), s));
  if (bs->n_rows) launch_count_v0(bs->rows.p, bs->pitch_words, bs->d_flat.p, k, M, bs->d_counts.p, s);
  else GPA_CUDA(cudaMemsetAsync(bs->d_counts.p, 0, M * sizeof(uint32_t), s));
  if (st) { st->kernel = GPA_KERNEL_V0; st->launches = 1; }
  finish_counts(bs, M, st);
}

// Transaction-tiled trie walk: cut the lexicographic candidate list into blocks (<= kTrieMaxCand
// candidates, <= kTrieMaxRows distinct rows), give every candidate its block-local row bytes and
// its shared-prefix length with the previous candidate of the same 32-candidate warp chunk.
void count_trie_batch(gpa_bitset* bs, const GroupedBatch& b, CountStats* st) {
  cudaStream_t s = bs->stream;
  const uint32_t k = b.k;
  const uint64_t M = b.size();
  const double tp0 = wall_ms();
  TriePlan P = plan_trie(b, bs->n_rows);
  const double tp1 = wall_ms();
  const auto& blocks = P.blocks;
  const auto& brows = P.rows;
  const auto& lrows = P.lrows;
  const auto& lcp = P.lcp;
  const uint32_t max_rows = P.max_rows;
  const uint32_t n_blocks = (uint32_t)blocks.size();
  const uint32_t n_stripes = (uint32_t)(bs->pitch_words / trie_stripe_words(k));
  uint32_t n_parts = std::max<uint32_t>(1, n_stripes / 64);
  const uint32_t want = (uint32_t)bs->n_sms * 2 * 3;
  if ((uint64_t)n_blocks * n_parts < want) n_parts = std::min<uint32_t>(n_stripes, (want + n_blocks - 1) / n_blocks);
  bs->d_tblocks.ensure(n_blocks, s);
  bs->d_trows.ensure(std::max<size_t>(brows.size(), 1), s);
  bs->d_lrows.ensure(M, s);
  bs->d_lcp.ensure(M, s);
  bs->d_counts.ensure(M, s);
  GPA_CUDA(cudaMemcpyAsync(bs->d_tblocks.p, blocks.data(), n_blocks * sizeof(TrieBlock), cudaMemcpyHostToDevice, s));
  GPA_CUDA(cudaMemcpyAsync(bs->d_trows.p, brows.data(), brows.size() * sizeof(uint32_t), cudaMemcpyHostToDevice, s));
  GPA_CUDA(cudaMemcpyAsync(bs->d_lrows.p, lrows.data(), M * sizeof(uint4), cudaMemcpyHostToDevice, s));
  GPA_CUDA(cudaMemcpyAsync(bs->d_lcp.p, lcp.data(), M, cudaMemcpyHostToDevice, s));
  GPA_CUDA(cudaMemsetAsync(bs->d_counts.p, 0, M * sizeof(uint32_t), s));
  GPA_CUDA(cudaEventRecord(ev_start(bs, st), s));
  if (bs->n_rows)
    launch_trie(k, bs->rows.p, bs->pitch_words, bs->d_tblocks.p, bs->d_trows.p, bs->d_lrows.p, bs->d_lcp.p,
                n_blocks, max_rows, n_parts, bs->d_counts.p, s);
  if (st) { st->kernel = GPA_KERNEL_TRIE; st->launches = 1; }
  const double tp2 = wall_ms();
  finish_counts(bs, M, st);
  if (trace_enabled())
    fprintf(stderr, "[gpa] k=%u trie: M=%llu blocks=%u max_rows=%u parts=%u plan %.2f ms, h2d+launch %.2f ms, "
            "kernel %.2f ms\n", k, (unsigned long long)M, n_blocks, max_rows, n_parts, tp1 - tp0, tp2 - tp1,
            st ? st->count_ms : -1.0);
}

}  // namespace

// ------------------------------------------------------------------ counting a device-resident batch

bool count_device_batch(gpa_bitset* bs, DeviceBatch& B, uint32_t kernel, DeviceScratch& scratch, CountStats* st) {
  cudaStream_t s = bs->stream;
  const uint32_t k = B.k, M = B.M, G = B.G;
  if (M == 0) return true;
  if (kernel == GPA_KERNEL_PROJ || kernel == GPA_KERNEL_FUSED) kernel = GPA_KERNEL_AUTO;
  if (kernel == GPA_KERNEL_V0 || bs->n_rows > kPlanMaxRows || k < 2) return false;
  if (kernel == GPA_KERNEL_AUTO || kernel == GPA_KERNEL_PAIRS || kernel == GPA_KERNEL_PAIRS_TC) {
    const double sib = (double)M / (double)std::max<uint32_t>(G, 1);
    kernel = (k <= kTrieMaxK && sib < auto_sibling_cut()) ? GPA_KERNEL_TRIE : GPA_KERNEL_PREFIX;
  }
  if (kernel == GPA_KERNEL_TRIE && k > kTrieMaxK) kernel = GPA_KERNEL_PREFIX;
  const double tp0 = wall_ms();
  bs->d_counts.ensure(M, s);
  if (kernel == GPA_KERNEL_PREFIX) {
    uint32_t* n_tasks = scratch.u32a(G, s);
    uint32_t* task_off = scratch.u32b(G, s);
    uint32_t* tot = scratch.u32c(1, s);
    launch_prefix_tasks(B.ext_off.p, G, n_tasks, nullptr, nullptr, bs->n_sms, s, false);
    device_exclusive_scan(n_tasks, task_off, G, tot, scratch, s);
    uint32_t T = 0;
    GPA_CUDA(cudaMemcpyAsync(&T, tot, 4, cudaMemcpyDeviceToHost, s));
    stream_wait(s);
    bs->d_tasks.ensure(T, s);
    launch_prefix_tasks(B.ext_off.p, G, nullptr, task_off, bs->d_tasks.p, bs->n_sms, s, true);
    GPA_CUDA(cudaMemsetAsync(bs->d_counts.p, 0, (size_t)M * 4, s));
    GPA_CUDA(cudaEventRecord(ev_start(bs, st), s));
    const uint32_t max_tasks = 1u << 20;
    uint32_t launches = 0;
    for (uint32_t t0 = 0; t0 < T; t0 += max_tasks) {
      launch_count_prefix(bs->rows.p, bs->pitch_words, B.prefix.p, k - 1, B.ext.p, bs->d_tasks.p + t0,
                          std::min(max_tasks, T - t0), bs->d_counts.p, s);
      ++launches;
    }
    if (st) { st->kernel = GPA_KERNEL_PREFIX; st->launches = launches; }
    finish_counts(bs, M, st);
    return true;
  }
  // trie: greedy blocks inside windows of 256 candidates (one CTA per window), one sync
  const uint32_t rmax = trie_max_rows(k);
  bs->d_cgroup.ensure(M, s);
  launch_cand_group(B.ext_off.p, G, bs->d_cgroup.p, bs->n_sms, s);
  const uint32_t window = kTrieMaxCand;
  const uint32_t n_win = (M + window - 1) / window;
  DBuf<uint3> d_recs;
  d_recs.alloc((size_t)n_win * window, s);
  uint32_t* d_nrec = scratch.u32d(n_win, s);
  launch_window_greedy(B.prefix.p, B.ext.p, bs->d_cgroup.p, k, bs->n_rows, M, window, rmax, d_recs.p, d_nrec, s);
  // block table on the device: scan of blocks per window, compaction, scan of rows per block
  uint32_t* d_woff = scratch.u32e(n_win, s);
  uint32_t* d_stats = scratch.u32f(4, s);   // [0] max rows, [1] #blocks, [2] #rows
  GPA_CUDA(cudaMemsetAsync(d_stats, 0, 16, s));
  device_exclusive_scan(d_nrec, d_woff, n_win, d_stats + 1, scratch, s);
  const uint32_t max_blocks = M;  // every block holds >= 1 candidate
  bs->d_tblocks.ensure(max_blocks, s);
  uint32_t* d_brows = scratch.u32g(max_blocks, s);
  uint32_t* d_roff = scratch.u32h(max_blocks, s);
  launch_compact_blocks(d_recs.p, d_nrec, d_woff, n_win, window, bs->d_tblocks.p, d_brows, d_stats, s);
  uint32_t st3[3] = {0, 0, 0};
  GPA_CUDA(cudaMemcpyAsync(st3, d_stats, 12, cudaMemcpyDeviceToHost, s));
  stream_wait(s);
  const uint32_t n_blocks = st3[1], max_rows = st3[0];
  device_exclusive_scan(d_brows, d_roff, n_blocks, d_stats + 2, scratch, s);
  launch_row_begin(d_roff, n_blocks, bs->d_tblocks.p, bs->n_sms, s);
  const uint32_t passes = 1;
  // total rows <= n_blocks * rmax
  const uint32_t rows_total = n_blocks * rmax;
  bs->d_trows.ensure(std::max<uint32_t>(rows_total, 1), s);
  bs->d_lrows.ensure(M, s);
  bs->d_lcp.ensure(M, s);
  launch_build_blocks(B.prefix.p, B.ext.p, bs->d_cgroup.p, k, bs->n_rows, bs->d_tblocks.p, n_blocks, bs->d_trows.p,
                      bs->d_lrows.p, bs->d_lcp.p, s);
  const uint32_t n_stripes = (uint32_t)(bs->pitch_words / trie_stripe_words(k));
  uint32_t n_parts = std::max<uint32_t>(1, n_stripes / 64);
  const uint32_t want = (uint32_t)bs->n_sms * 2 * 3;
  if ((uint64_t)n_blocks * n_parts < want) n_parts = std::min<uint32_t>(n_stripes, (want + n_blocks - 1) / n_blocks);
  GPA_CUDA(cudaMemsetAsync(bs->d_counts.p, 0, (size_t)M * 4, s));
  const double tp1 = wall_ms();
  GPA_CUDA(cudaEventRecord(ev_start(bs, st), s));
  launch_trie(k, bs->rows.p, bs->pitch_words, bs->d_tblocks.p, bs->d_trows.p, bs->d_lrows.p, bs->d_lcp.p,
              n_blocks, max_rows, n_parts, bs->d_counts.p, s);
  if (st) { st->kernel = GPA_KERNEL_TRIE; st->launches = 1; }
  finish_counts(bs, M, st);
  if (trace_enabled())
    fprintf(stderr, "[gpa] k=%u trie (device plan, %u passes): M=%u blocks=%u max_rows=%u parts=%u plan %.2f ms, "
            "kernel %.2f ms\n", k, passes, M, n_blocks, max_rows, n_parts, tp1 - tp0, st ? st->count_ms : -1.0);
  return true;
}

void count_grouped(gpa_bitset* bs, const GroupedBatch& b, uint32_t kernel, CountStats* st) {
  cudaStream_t s = bs->stream;
  const uint64_t M = b.size(), G = b.groups();
  const uint32_t km1 = b.k - 1;
  if (M == 0) return;
  if (kernel == GPA_KERNEL_PROJ || kernel == GPA_KERNEL_FUSED) kernel = GPA_KERNEL_AUTO;
  if (kernel == GPA_KERNEL_AUTO || kernel == GPA_KERNEL_PAIRS || kernel == GPA_KERNEL_PAIRS_TC) {
    // grouped batches: large sibling groups amortise the (k-1)-row prefix well in the streaming
    // prefix kernel (measured: T40I10D10M k = 3, 4.6 siblings / group); small groups (deep
    // generations, ~2 siblings) need the trie walk's reuse across groups
    const double sib = (double)M / (double)std::max<uint64_t>(G, 1);
    kernel = (b.k >= 2 && b.k <= kTrieMaxK && sib < auto_sibling_cut()) ? GPA_KERNEL_TRIE : GPA_KERNEL_PREFIX;
  }
  if (kernel == GPA_KERNEL_TRIE) {
    if (b.k >= 2 && b.k <= kTrieMaxK) {
      count_trie_batch(bs, b, st);
      return;
    }
    kernel = GPA_KERNEL_PREFIX;
  }
  if (kernel == GPA_KERNEL_V0 || km1 == 0) {
    std::vector<uint32_t> flat(M * b.k);
    for (uint64_t g = 0; g < G; ++g)
      for (uint64_t j = b.ext_off[g]; j < b.ext_off[g + 1]; ++j) {
        std::copy(b.prefix.begin() + g * km1, b.prefix.begin() + (g + 1) * km1, flat.begin() + j * b.k);
        flat[j * b.k + km1] = b.ext[j];
      }
    count_flat_v0(bs, flat, b.k, M, st);
    return;
  }
  GPA_REQUIRE(G < (1ull << 32) && M < (1ull << 32), GPA_ERR_INVALID, "candidate batch too large");
  // tasks: each group split into chunks of <= kPrefixMaxSiblings siblings
  std::vector<PrefixTask> tasks;
  tasks.reserve(M / 8 + G);
  for (uint64_t g = 0; g < G; ++g)
    for (uint64_t j = b.ext_off[g]; j < b.ext_off[g + 1]; j += kPrefixMaxSiblings) {
      uint32_t n = (uint32_t)std::min<uint64_t>(kPrefixMaxSiblings, b.ext_off[g + 1] - j);
      tasks.push_back(PrefixTask{(uint32_t)g, (uint32_t)j, n, 0});
    }
  bs->d_prefix.ensure(b.prefix.size(), s);
  bs->d_ext.ensure(M, s);
  bs->d_tasks.ensure(tasks.size(), s);
  bs->d_counts.ensure(M, s);
  GPA_CUDA(cudaMemcpyAsync(bs->d_prefix.p, b.prefix.data(), b.prefix.size() * sizeof(uint32_t), cudaMemcpyHostToDevice, s));
  GPA_CUDA(cudaMemcpyAsync(bs->d_ext.p, b.ext.data(), M * sizeof(uint32_t), cudaMemcpyHostToDevice, s));
  GPA_CUDA(cudaMemcpyAsync(bs->d_tasks.p, tasks.data(), tasks.size() * sizeof(PrefixTask), cudaMemcpyHostToDevice, s));
  GPA_CUDA(cudaMemsetAsync(bs->d_counts.p, 0, M * sizeof(uint32_t), s));
  GPA_CUDA(cudaEventRecord(ev_start(bs, st), s));
  // a task index must fit the kernel's 32-bit grid decode: launch in slices of tasks if needed
  const uint64_t max_tasks = 1u << 20;
  uint32_t launches = 0;
  for (uint64_t t0 = 0; t0 < tasks.size(); t0 += max_tasks) {
    uint32_t nt = (uint32_t)std::min<uint64_t>(max_tasks, tasks.size() - t0);
    launch_count_prefix(bs->rows.p, bs->pitch_words, bs->d_prefix.p, km1, bs->d_ext.p, bs->d_tasks.p + t0, nt,
                        bs->d_counts.p, s);
    ++launches;
  }
  if (st) { st->kernel = GPA_KERNEL_PREFIX; st->launches = launches; }
  finish_counts(bs, M, st);
}

void count_all_pairs(gpa_bitset* bs, uint32_t kernel, CountStats* st) {
  cudaStream_t s = bs->stream;
  const uint64_t n = l1_size(bs);
  const uint64_t M = n * (n - 1) / 2;
  if (n < 2) return;
  const bool sub = bs->l1_sub;   // L_1 is a subset of the rows
  if (kernel == GPA_KERNEL_AUTO || kernel == GPA_KERNEL_PROJ || kernel == GPA_KERNEL_FUSED) kernel = GPA_KERNEL_PAIRS_TC;
  if (kernel != GPA_KERNEL_PAIRS && kernel != GPA_KERNEL_PAIRS_TC) {
    GroupedBatch b;
    b.k = 2;
    b.ext_off.push_back(0);
    auto row = [&](uint64_t i) { return sub ? bs->l1[i] : (uint32_t)i; };
    for (uint64_t a = 0; a + 1 < n; ++a) {
      b.prefix.push_back(row(a));
      for (uint64_t c = a + 1; c < n; ++c) b.ext.push_back(row(c));
      b.ext_off.push_back(b.ext.size());
    }
    count_grouped(bs, b, kernel, st);
    return;
  }
  if (kernel == GPA_KERNEL_PAIRS && !bs->tmap_ready) {
    make_pairs_tensor_map(bs->tmap, bs->rows.p, bs->n_rows, bs->pitch_words);
    bs->tmap_ready = true;
  }
  // the pair Gram over every row, then (L_1 a subset) the L_1 pairs gathered out of it
  const uint64_t P = (uint64_t)bs->n_rows * (bs->n_rows - 1) / 2;
  uint32_t* dst = bs->d_counts.p;
  bs->d_counts.ensure(M, s);
  dst = bs->d_counts.p;
  if (sub) {
    bs->d_pairs_all.ensure(P, s);
    dst = bs->d_pairs_all.p;
    if (bs->d_l1.n < n) {
      bs->d_l1.alloc(n, s);
      GPA_CUDA(cudaMemcpyAsync(bs->d_l1.p, bs->l1.data(), n * 4, cudaMemcpyHostToDevice, s));
    }
  }
  GPA_CUDA(cudaMemsetAsync(dst, 0, (sub ? P : M) * sizeof(uint32_t), s));
  GPA_CUDA(cudaEventRecord(ev_start(bs, st), s));
  if (kernel == GPA_KERNEL_PAIRS_TC)
    launch_count_pairs_tc(bs->rows.p, bs->pitch_words, bs->n_rows, 0, bs->pitch_words, dst, bs->n_sms, s);
  else
    launch_count_pairs(bs->tmap, bs->n_rows, 0, bs->pitch_words, dst, bs->n_sms, s);
  if (sub) launch_pairs_subset(dst, bs->n_rows, bs->d_l1.p, (uint32_t)n, bs->d_counts.p, bs->n_sms, s);
  if (st) { st->kernel = kernel; st->launches = sub ? 2 : 1; }
  finish_counts(bs, M, st);
}

}  // namespace gpa

// ---------------------------------------------------------------- C ABI: options, threshold, bitset

extern "C" void gpa_options_default(gpa_options* opt) {
  if (!opt) return;
  memset(opt, 0, sizeof(*opt));
  opt->count_kernel = GPA_KERNEL_AUTO;
  opt->device = -1;
}

extern "C" uint64_t gpa_min_count(uint64_t n_tx, uint64_t num, uint64_t den) {
  if (den == 0) return 0;
  unsigned __int128 q = ((unsigned __int128)n_tx * num + den - 1) / den;
  if (q > UINT64_MAX) q = UINT64_MAX;
  return q < 1 ? 1 : (uint64_t)q;
}

extern "C" gpa_status gpa_bitset_create(const gpa_tx_csr* db, uint32_t row_min_count, const gpa_dist* dist,
                                        const gpa_options* opt, gpa_bitset** out) {
  return gpa::guard([&] {
    GPA_REQUIRE(out, GPA_ERR_INVALID, "out is NULL");
    gpa::DistScope scope(dist);
    *out = gpa::bitset_build(db, row_min_count, dist, opt);
  });
}

extern "C" gpa_status gpa_bitset_destroy(gpa_bitset* bs) {
  return gpa::guard([&] { gpa::bitset_free(bs); });
}

extern "C" gpa_status gpa_bitset_info(const gpa_bitset* bs, uint64_t* n_tx_local, uint64_t* n_tx_global,
                                      uint32_t* n_rows, uint64_t* row_pitch_bytes) {
  return gpa::guard([&] {
    GPA_REQUIRE(bs, GPA_ERR_INVALID, "bitset is NULL");
    if (n_tx_local) *n_tx_local = bs->n_tx_local;
    if (n_tx_global) *n_tx_global = bs->n_tx_global;
    if (n_rows) *n_rows = bs->n_rows;
    if (row_pitch_bytes) *row_pitch_bytes = bs->pitch_words * 4;
  });
}

extern "C" gpa_status gpa_bitset_item_counts(const gpa_bitset* bs, uint32_t* counts_out) {
  return gpa::guard([&] {
    GPA_REQUIRE(bs && counts_out, GPA_ERR_INVALID, "NULL argument");
    std::copy(bs->item_counts.begin(), bs->item_counts.end(), counts_out);
  });
}

extern "C" gpa_status gpa_bitset_rows(const gpa_bitset* bs, uint32_t* item_of_row_out) {
  return gpa::guard([&] {
    GPA_REQUIRE(bs && (item_of_row_out || bs->n_rows == 0), GPA_ERR_INVALID, "NULL argument");
    std::copy(bs->item_of_row.begin(), bs->item_of_row.end(), item_of_row_out);
  });
}

extern "C" gpa_status gpa_bitset_export(const gpa_bitset* bs, uint32_t* host_out) {
  return gpa::guard([&] {
    GPA_REQUIRE(bs && (host_out || bs->n_rows == 0), GPA_ERR_INVALID, "NULL argument");
    if (!bs->n_rows) return;
    gpa::use_device(bs->device);
    GPA_CUDA(cudaMemcpyAsync(host_out, bs->rows.p, (size_t)bs->n_rows * bs->pitch_words * 4, cudaMemcpyDeviceToHost,
                             bs->stream));
    gpa::stream_wait(bs->stream);
  });
}

extern "C" gpa_status gpa_count(gpa_bitset* bs, const uint32_t* cand, uint32_t k, uint64_t M, uint32_t kernel,
                                uint32_t* counts_out) {
  return gpa::guard([&] {
    GPA_REQUIRE(bs, GPA_ERR_INVALID, "bitset is NULL");
    GPA_REQUIRE(k >= 1 && k <= GPA_MAX_K, GPA_ERR_INVALID, "k must be in [1, %u]", GPA_MAX_K);
    GPA_REQUIRE(kernel <= GPA_KERNEL_FUSED, GPA_ERR_INVALID, "unknown kernel %u", kernel);
    if (M == 0) return;
    GPA_REQUIRE(cand && counts_out, GPA_ERR_INVALID, "NULL argument");
    GPA_REQUIRE(M <= (UINT64_MAX / 8) / k && M < (1ull << 32), GPA_ERR_INVALID, "M * k overflows");
    gpa::dist_check(bs->dist);
    gpa::use_device(bs->device);
    gpa::DistScope scope(bs->dist);
    // validate + translate to row ids; with dist the verdict is agreed across ranks before the
    // counting collective (a rank-local rejection must not strand the others)
    std::vector<uint32_t> rows(M * k);
    uint32_t verdict[1] = {GPA_OK};
    std::string why;
    try {
      for (uint64_t m = 0; m < M; ++m) {
        for (uint32_t j = 0; j < k; ++j) {
          const uint32_t it = cand[m * k + j];
          GPA_REQUIRE(it < bs->n_items, GPA_ERR_INVALID, "candidate %llu: item %u >= n_items", (unsigned long long)m, it);
          GPA_REQUIRE(j == 0 || it > cand[m * k + j - 1], GPA_ERR_INVALID,
                      "candidate %llu is not strictly increasing", (unsigned long long)m);
          const int32_t r = bs->row_of_item[it];
          GPA_REQUIRE(r >= 0, GPA_ERR_RANGE, "item %u has no bitset row", it);
          rows[m * k + j] = (uint32_t)r;
        }
      }
    } catch (const gpa::Error& e) {
      verdict[0] = e.status;
      why = e.msg;
    }
    gpa::dist_agree_max(bs->dist, verdict, 1);
    if (verdict[0] != GPA_OK) {
      if (!why.empty()) gpa::fail((gpa_status)verdict[0], "%s", why.c_str());
      gpa::fail((gpa_status)verdict[0], "invalid candidates on another rank");
    }
    uint32_t kern = kernel == GPA_KERNEL_AUTO ? bs->opt.count_kernel : kernel;
    if (kern == GPA_KERNEL_PROJ || kern == GPA_KERNEL_FUSED) kern = GPA_KERNEL_AUTO;  // gpa_mine's level structure
    if (k == 1) kern = GPA_KERNEL_V0;
    if (kern == GPA_KERNEL_AUTO)
      kern = (k == 2 && (double)M * 8 >= (double)bs->n_rows * bs->n_rows) ? GPA_KERNEL_PAIRS_TC
             : (k <= gpa::kTrieMaxK ? GPA_KERNEL_TRIE : GPA_KERNEL_PREFIX);
    if ((kern == GPA_KERNEL_PAIRS || kern == GPA_KERNEL_PAIRS_TC) && k != 2)
      kern = k <= gpa::kTrieMaxK ? GPA_KERNEL_TRIE : GPA_KERNEL_PREFIX;
    if (kern == GPA_KERNEL_PAIRS || kern == GPA_KERNEL_PAIRS_TC) {
      gpa::count_all_pairs(bs, kern, nullptr);
      const uint64_t n = bs->n_rows, P = n * (n - 1) / 2;
      std::vector<uint32_t> all(P);
      if (P) {
        GPA_CUDA(cudaMemcpyAsync(all.data(), bs->d_counts.p, P * 4, cudaMemcpyDeviceToHost, bs->stream));
        gpa::stream_wait(bs->stream);
      }
      for (uint64_t m = 0; m < M; ++m) counts_out[m] = all[gpa::pair_index(rows[2 * m], rows[2 * m + 1], n)];
      return;
    }
    if (kern == GPA_KERNEL_V0) {
      gpa::GroupedBatch b;  // V0 path takes the flat batch in caller order: one group per candidate
      b.k = k;
      b.ext_off.resize(M + 1);
      b.prefix.resize(M * (k - 1));
      b.ext.resize(M);
      for (uint64_t m = 0; m < M; ++m) {
        std::copy(rows.begin() + m * k, rows.begin() + m * k + k - 1, b.prefix.begin() + m * (k - 1));
        b.ext[m] = rows[m * k + k - 1];
        b.ext_off[m] = m;
      }
      b.ext_off[M] = M;
      gpa::count_grouped(bs, b, GPA_KERNEL_V0, nullptr);
      GPA_CUDA(cudaMemcpyAsync(counts_out, bs->d_counts.p, M * 4, cudaMemcpyDeviceToHost, bs->stream));
      gpa::stream_wait(bs->stream);
      return;
    }
    // PREFIX / TRIE: group by (k-1)-prefix (sort candidate indices lexicographically)
    std::vector<uint64_t> order(M);
    std::iota(order.begin(), order.end(), 0);
    std::sort(order.begin(), order.end(), [&](uint64_t a, uint64_t b) {
      return std::lexicographical_compare(rows.begin() + a * k, rows.begin() + a * k + k, rows.begin() + b * k,
                                          rows.begin() + b * k + k);
    });
    gpa::GroupedBatch b;
    b.k = k;
    b.ext.resize(M);
    for (uint64_t i = 0; i < M; ++i) {
      const uint64_t m = order[i];
      const bool new_group = i == 0 || !std::equal(rows.begin() + m * k, rows.begin() + m * k + k - 1,
                                                    rows.begin() + order[i - 1] * k);
      if (new_group) {
        b.ext_off.push_back(i);
        b.prefix.insert(b.prefix.end(), rows.begin() + m * k, rows.begin() + m * k + k - 1);
      }
      b.ext[i] = rows[m * k + k - 1];
    }
    b.ext_off.push_back(M);
    gpa::count_grouped(bs, b, kern, nullptr);
    std::vector<uint32_t> sorted(M);
    GPA_CUDA(cudaMemcpyAsync(sorted.data(), bs->d_counts.p, M * 4, cudaMemcpyDeviceToHost, bs->stream));
    gpa::stream_wait(bs->stream);
    for (uint64_t i = 0; i < M; ++i) counts_out[order[i]] = sorted[i];
  });
}
