// Overlapped ingest for host-resident input (gpa_mine end to end).
//
// Copying the horizontal database to the GPU (the paper's "copied ... to graphic memory",
// P18@451/P18@755) costs as much as a third of a mining pass over PCIe.  Support counting is a
// sum over transactions, so generation 2 can be counted chunk by chunk WHILE the next chunk of
// transactions is still in flight: the CSR is split into ~8 transaction chunks (multiples of 8,192
// transactions = whole bitset stripes); a copy stream uploads chunk c+1 while the compute stream
// runs, for chunk c, the validation + histogram kernel, the static-bitset build and the tiled pair
// kernel over the chunk's words.
//
// The rows of the bitset must be chosen before the global item counts are known.  After chunk 0
// the rows are the items whose chunk-0 frequency, extrapolated, reaches half the threshold
// (R0 -- a superset of L_1 with high probability).  At the end: if L_1 is contained in R0, the L_1
// rows are gathered out of the R0 bitset and the L_1 pairs out of the R0 pair counts (exact:
// counts are sums over transactions, the extra rows only cost work); otherwise the bitset is
// rebuilt for L_1 from the device copy of the CSR and generation 2 is counted afresh.  Either way
// the result is identical to the sequential path (same counts, same rows).
#include <algorithm>
#include <array>
#include <cstdlib>
#include <utility>
#include <map>

#include "internal.h"
#include "pool.h"

namespace gpa {

namespace {
constexpr uint64_t kIngestAlign = 8192;   // transactions: one bitset stripe (256 words)
constexpr uint32_t kIngestChunks = 8;

// Bit-packed upload of the item ids (the PCIe transfer bounds gpa_mine on host input): with
// n_items <= 2^16 every id fits in b = ceil(log2 n_items) bits, so host threads pack a chunk's
// items into b-bit fields (32 items = b whole words per block: blocks pack independently) in a
// page-locked staging buffer, the copy stream moves b/32 of the bytes, and unpack.cu widens them
// in place in the device CSR.  An id >= 2^b (invalid input) sends that chunk as raw u32, so the
// validation kernel sees and rejects it as before.  GPA_NO_PACKED_UPLOAD=1 disables it.
uint32_t pack_bits(uint32_t n_items) {
  if (const char* e = getenv("GPA_NO_PACKED_UPLOAD"))
    if (*e && *e != '0') return 0;
  uint32_t b = 1;
  while (b < 32 && (1ull << b) < n_items) ++b;
  return b <= 16 ? b : 0;
}

struct PackStage {   // per thread and device: three host staging buffers + one device buffer
  uint32_t* h[3] = {nullptr, nullptr, nullptr};
  cudaEvent_t ev[3] = {nullptr, nullptr, nullptr};   // the H2D out of h[i] done
  bool pending[3] = {false, false, false};
  size_t cap = 0;                                    // words per buffer
  PBuf<uint32_t> d;
  void ensure(size_t words) {
    if (!ev[0])
      for (auto& e : ev) GPA_CUDA(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
    if (words <= cap) return;
    for (int i = 0; i < 3; ++i) {
      if (pending[i]) GPA_CUDA(cudaEventSynchronize(ev[i]));
      pending[i] = false;
      if (h[i]) cudaFreeHost(h[i]);
      h[i] = nullptr;
    }
    cap = 0;
    for (auto& x : h) GPA_CUDA(cudaHostAlloc(reinterpret_cast<void**>(&x), words * 4, cudaHostAllocDefault));
    cap = words;
    d.ensure(words);
  }
  ~PackStage() {
    for (int i = 0; i < 3; ++i) {
      if (pending[i]) cudaEventSynchronize(ev[i]);
      if (h[i]) cudaFreeHost(h[i]);
      if (ev[i]) cudaEventDestroy(ev[i]);
    }
  }
};
PackStage& pack_stage(int device) {
  thread_local std::map<int, PackStage> m;
  return m[device];
}

// one block of 32 ids -> B words (B a compile-time constant: straight-line shifts and ORs)
template <uint32_t B>
inline uint32_t pack_block(const uint32_t* __restrict__ src, uint32_t* __restrict__ dst) {
  uint32_t orv = 0;
  uint64_t acc = 0;
  uint32_t nb = 0, k = 0;
#pragma GCC unroll 32
  for (uint32_t i = 0; i < 32; ++i) {
    const uint32_t v = src[i];
    orv |= v;
    acc |= (uint64_t)v << nb;
    nb += B;
    if (nb >= 32) {
      dst[k++] = (uint32_t)acc;
      acc >>= 32;
      nb -= 32;
    }
  }
  return orv;
}

template <uint32_t B>
uint32_t pack_range(const uint32_t* items, uint64_t n, uint64_t blk0, uint64_t blk1, uint32_t* words) {
  uint32_t orv = 0;
  for (uint64_t blk = blk0; blk < blk1; ++blk) {
    const uint64_t j0 = blk * 32;
    if (j0 + 32 <= n) {
      orv |= pack_block<B>(items + j0, words + blk * B);
    } else {   // the ragged last block: zero-padded copy
      uint32_t tmp[32] = {};
      for (uint64_t j = j0; j < n; ++j) tmp[j - j0] = items[j];
      orv |= pack_block<B>(tmp, words + blk * B);
    }
  }
  return orv;
}

using PackFn = uint32_t (*)(const uint32_t*, uint64_t, uint64_t, uint64_t, uint32_t*);
template <uint32_t... Bs>
constexpr std::array<PackFn, sizeof...(Bs)> pack_table(std::integer_sequence<uint32_t, Bs...>) {
  return {&pack_range<Bs + 1>...};
}

// items[0, n) -> b-bit fields in words (ceil(n / 32) * b words); returns false if an id >= 2^b
bool pack_items(const uint32_t* items, uint64_t n, uint32_t b, uint32_t* words) {
  static constexpr auto table = pack_table(std::make_integer_sequence<uint32_t, 16>{});
  const PackFn fn = table[b - 1];
  const uint64_t nblk = (n + 31) / 32;
  const size_t T = std::max<size_t>(1, std::min<uint64_t>(pool_threads() * 4, (nblk + 1023) / 1024));
  std::vector<uint32_t> ors(T, 0);
  parallel_for(T, [&](size_t t) { ors[t] = fn(items, n, nblk * t / T, nblk * (t + 1) / T, words); });
  uint32_t o = 0;
  for (uint32_t v : ors) o |= v;
  return (o >> b) == 0;
}
}  // namespace

bool ingest_overlap_eligible(const gpa_tx_csr* db) {
  return db && db->memory == GPA_MEM_HOST && db->n_tx >= kIngestChunks * 4 * kIngestAlign && db->n_items >= 2 &&
         db->n_items <= 16384 && db->offsets && db->items;
}

std::vector<uint64_t> ingest_cuts(uint64_t n_tx) {
  uint64_t ct = (n_tx + kIngestChunks - 1) / kIngestChunks;
  ct = (ct + kIngestAlign - 1) / kIngestAlign * kIngestAlign;
  std::vector<uint64_t> cut;
  for (uint64_t t = 0; t < n_tx; t += ct) cut.push_back(t);
  cut.push_back(n_tx);
  return cut;
}

bool agree_input(const gpa_tx_csr* db, const gpa_dist* dist, bool want_overlap) {
  enum : uint32_t { kBad = 1, kNoOverlap = 2 };
  uint32_t flags = 0;
  std::string why;
  auto bad = [&](const char* m) {
    if (!(flags & kBad)) why = m;
    flags |= kBad;
  };
  if (!db) {
    bad("db is NULL");
  } else if (db->memory != GPA_MEM_HOST && db->memory != GPA_MEM_DEVICE) {
    bad("db->memory must be GPA_MEM_HOST or GPA_MEM_DEVICE");
  } else if (!db->offsets) {
    bad("db->offsets is NULL");
  } else if (db->memory == GPA_MEM_HOST) {
    if (db->offsets[0] != 0) bad("offsets[0] must be 0");
    else if (db->offsets[db->n_tx] > 0 && !db->items) bad("db->items is NULL");
    else {
      const std::vector<uint64_t> cut = ingest_cuts(db->n_tx);   // the upload sizes come from these
      for (size_t c = 0; c + 1 < cut.size(); ++c)
        if (db->offsets[cut[c + 1]] < db->offsets[cut[c]]) bad("offsets are not non-decreasing");
    }
  } else if (db->n_tx) {
    uint64_t first = 0;
    GPA_CUDA(cudaMemcpy(&first, db->offsets, sizeof(uint64_t), cudaMemcpyDeviceToHost));
    if (first != 0) bad("offsets[0] must be 0");
  }
  if (!(want_overlap && ingest_overlap_eligible(db))) flags |= kNoOverlap;
  const uint32_t n_items = db ? db->n_items : 0;
  uint32_t v[3] = {flags, n_items, ~n_items};   // max of n_items and of its complement: max and min
  dist_agree_max(dist, v, 3);
  if (v[0] & kBad) {
    if (flags & kBad) fail(GPA_ERR_INVALID, "%s", why.c_str());
    fail(GPA_ERR_INVALID, "invalid input on another rank");
  }
  GPA_REQUIRE(v[1] == n_items && ~v[2] == n_items, GPA_ERR_INVALID, "ranks disagree on n_items (%u .. %u)", ~v[2],
              v[1]);
  return !(v[0] & kNoOverlap);
}

gpa_bitset* bitset_build_overlapped(const gpa_tx_csr* db, uint64_t row_min_count, const gpa_dist* dist,
                                    const gpa_options* opt_in, bool* pairs_ready, CountStats* pair_stats) {
  *pairs_ready = false;
  gpa_options opt;
  gpa_options_default(&opt);
  if (opt_in) opt = *opt_in;
  dist_check(dist);
  DeviceInfo di = use_device(dist ? dist->device : opt.device);
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
  cudaStream_t cs = nullptr;
  GPA_CUDA(cudaStreamCreateWithFlags(&cs, cudaStreamNonBlocking));
  struct StreamGuard {
    cudaStream_t st;
    ~StreamGuard() { if (st) { cudaStreamSynchronize(st); cudaStreamDestroy(st); } }
  } cs_guard{cs};

  const double t0 = wall_ms();
  const uint64_t n_tx = db->n_tx;
  const uint32_t n_items = db->n_items;
  const uint64_t nnz = db->offsets[n_tx];
  bs->pitch_words = pitch_words_for(n_tx);

  // chunk plan (agree_input checked offsets[0] and the monotonicity at the cuts on every rank)
  const std::vector<uint64_t> cut = ingest_cuts(n_tx);
  const size_t C = cut.size() - 1;

  DBuf<uint64_t> d_off;
  DBuf<uint32_t> d_items, d_hist, d_flags;
  DBuf<uint64_t> d_ntx;
  d_off.alloc(n_tx + 1, s);
  d_items.alloc(std::max<uint64_t>(nnz, 1), s);
  d_hist.alloc(n_items, s);
  d_flags.alloc(1, s);
  d_ntx.alloc(1, s);
  GPA_CUDA(cudaMemsetAsync(d_hist.p, 0, n_items * 4, s));
  GPA_CUDA(cudaMemsetAsync(d_flags.p, 0, 4, s));
  GPA_CUDA(cudaMemcpyAsync(d_ntx.p, &bs->n_tx_local, 8, cudaMemcpyHostToDevice, s));
  stream_wait(s);  // the copy stream writes into these allocations
  std::vector<cudaEvent_t> up(C, nullptr);
  struct EvGuard {
    std::vector<cudaEvent_t>& v;
    ~EvGuard() { for (auto e : v) if (e) cudaEventDestroy(e); }
  } ev_guard{up};
  const uint32_t pbits = pack_bits(n_items);
  PackStage* ps = nullptr;
  if (pbits) {
    uint64_t max_items = 0;
    for (size_t c = 0; c < C; ++c) max_items = std::max<uint64_t>(max_items, db->offsets[cut[c + 1]] - db->offsets[cut[c]]);
    ps = &pack_stage(bs->device);
    ps->ensure((max_items + 31) / 32 * pbits + 1);
  }
  uint64_t packed_bytes = 0;
  const uint32_t raw_every = [] {
    const char* e = getenv("GPA_PACK_RAW_EVERY");
    return e ? (uint32_t)atoi(e) : 4u;   // measured (T40I10D10M, per call): all packed 40-42 ms, every 3rd raw 36.3, every 4th raw 35
  }();
  auto upload = [&](size_t c) {
    const uint64_t a = cut[c], b = cut[c + 1];
    const uint64_t ia = db->offsets[a], ib = db->offsets[b];
    GPA_CUDA(cudaMemcpyAsync(d_off.p + a, db->offsets + a, (b - a + 1) * 8, cudaMemcpyHostToDevice, cs));
    bool raw = ib > ia;
    // every raw_every-th chunk (from chunk 0) goes raw: the copy engine has PCIe bandwidth to spare
    // while the host packs (packing is host-bound at ~70 GB/s, the packed stream needs ~20 GB/s of
    // PCIe), so the two run side by side
    if (ib > ia && ps && (raw_every == 0 || c % raw_every != 0)) {
      const int slot = (int)(c % 3);
      if (ps->pending[slot]) GPA_CUDA(cudaEventSynchronize(ps->ev[slot]));   // chunk c - 3's H2D is done
      ps->pending[slot] = false;
      const uint64_t n = ib - ia, words = (n + 31) / 32 * pbits;
      if (pack_items(db->items + ia, n, pbits, ps->h[slot])) {
        GPA_CUDA(cudaMemcpyAsync(ps->d.p, ps->h[slot], words * 4, cudaMemcpyHostToDevice, cs));
        GPA_CUDA(cudaEventRecord(ps->ev[slot], cs));
        ps->pending[slot] = true;
        // (the single device buffer is reused by the next chunk's H2D after this kernel: stream order)
        launch_unpack_items(ps->d.p, n, pbits, d_items.p + ia, bs->n_sms, cs);
        packed_bytes += words * 4;
        raw = false;
      }
    }
    if (raw) {
      GPA_CUDA(cudaMemcpyAsync(d_items.p + ia, db->items + ia, (ib - ia) * 4, cudaMemcpyHostToDevice, cs));
      packed_bytes += (ib - ia) * 4;
    }
    GPA_CUDA(cudaEventCreateWithFlags(&up[c], cudaEventDisableTiming));
    GPA_CUDA(cudaEventRecord(up[c], cs));
  };

  // ---- chunk 0: upload, histogram, choose the rows R0
  upload(0);
  if (C > 1) upload(1);
  GPA_CUDA(cudaStreamWaitEvent(s, up[0], 0));
  launch_hist_validate_range(d_off.p, d_items.p, cut[0], cut[1], nnz, n_items, d_hist.p, d_flags.p, bs->n_sms, s);
  DBuf<uint32_t> d_h0;
  d_h0.alloc(n_items, s);
  GPA_CUDA(cudaMemcpyAsync(d_h0.p, d_hist.p, n_items * 4, cudaMemcpyDeviceToDevice, s));
  DBuf<uint64_t> d_n0;
  d_n0.alloc(1, s);
  const uint64_t n0_local = cut[1] - cut[0];
  GPA_CUDA(cudaMemcpyAsync(d_n0.p, &n0_local, 8, cudaMemcpyHostToDevice, s));
  allreduce_sum_u32(dist, d_h0.p, n_items, s);  // every rank chooses the same R0
  allreduce_sum_u64(dist, d_n0.p, 1, s);
  allreduce_sum_u64(dist, d_ntx.p, 1, s);
  std::vector<uint32_t> h0(n_items);
  uint64_t n0 = 0, n_global = 0;
  GPA_CUDA(cudaMemcpyAsync(h0.data(), d_h0.p, n_items * 4, cudaMemcpyDeviceToHost, s));
  GPA_CUDA(cudaMemcpyAsync(&n0, d_n0.p, 8, cudaMemcpyDeviceToHost, s));
  GPA_CUDA(cudaMemcpyAsync(&n_global, d_ntx.p, 8, cudaMemcpyDeviceToHost, s));
  stream_wait(s);
  // R0: chunk-0 count >= half the threshold scaled to the chunk (h0 * N * 2 >= theta * n0)
  std::vector<uint32_t> r0_items;
  std::vector<int32_t> r0_of_item(n_items, -1);
  for (uint32_t i = 0; i < n_items; ++i)
    if (h0[i] > 0 && (unsigned __int128)h0[i] * n_global * 2 >= (unsigned __int128)row_min_count * n0) {
      r0_of_item[i] = (int32_t)r0_items.size();
      r0_items.push_back(i);
    }
  const uint32_t nr0 = (uint32_t)r0_items.size();
  DBuf<int32_t> d_r0map;
  DBuf<uint32_t> d_r0rows, d_r0pairs;
  d_r0map.alloc(n_items, s);
  GPA_CUDA(cudaMemcpyAsync(d_r0map.p, r0_of_item.data(), n_items * 4, cudaMemcpyHostToDevice, s));
  const uint64_t P0 = (uint64_t)nr0 * (nr0 ? nr0 - 1 : 0) / 2;
  alignas(64) unsigned char tmap0[128];
  // generation 2 on the tensor cores unless the caller pinned the CUDA-core pair kernel
  const bool pairs_tc = bs->opt.count_kernel != GPA_KERNEL_PAIRS;
  if (nr0) {
    d_r0rows.alloc((size_t)nr0 * bs->pitch_words, s);
    d_r0pairs.alloc(std::max<uint64_t>(P0, 1), s);
    GPA_CUDA(cudaMemsetAsync(d_r0pairs.p, 0, std::max<uint64_t>(P0, 1) * 4, s));
    if (nr0 >= 2 && !pairs_tc) make_pairs_tensor_map(tmap0, d_r0rows.p, nr0, bs->pitch_words);
  }
  double pairs_ms = 0;
  uint32_t pair_launches = 0;
  std::vector<cudaEvent_t> pe(2 * C, nullptr);
  struct EvGuard2 {
    std::vector<cudaEvent_t>& v;
    ~EvGuard2() { for (auto e : v) if (e) cudaEventDestroy(e); }
  } pe_guard{pe};

  // ---- all chunks: (upload c+1 in flight) histogram, bitset build over R0, generation-2 pairs
  for (size_t c = 0; c < C; ++c) {
    if (c + 2 < C) upload(c + 2);
    if (c > 0) {
      GPA_CUDA(cudaStreamWaitEvent(s, up[c], 0));
      launch_hist_validate_range(d_off.p, d_items.p, cut[c], cut[c + 1], nnz, n_items, d_hist.p, d_flags.p, bs->n_sms, s);
    }
    if (nr0) {
      launch_bitset_build(d_off.p, d_items.p, n_tx, nnz, d_r0map.p, n_items, nr0, bs->pitch_words, d_r0rows.p, cut[c],
                          cut[c + 1], s);
      if (nr0 >= 2) {
        GPA_CUDA(cudaEventCreate(&pe[2 * c]));
        GPA_CUDA(cudaEventCreate(&pe[2 * c + 1]));
        GPA_CUDA(cudaEventRecord(pe[2 * c], s));
        const uint64_t w0 = cut[c] / 32, w1 = c + 1 == C ? bs->pitch_words : cut[c + 1] / 32;
        if (pairs_tc)
          launch_count_pairs_tc(d_r0rows.p, bs->pitch_words, nr0, w0, w1, d_r0pairs.p, bs->n_sms, s);
        else
          launch_count_pairs(tmap0, nr0, w0, w1, d_r0pairs.p, bs->n_sms, s);
        GPA_CUDA(cudaEventRecord(pe[2 * c + 1], s));
        ++pair_launches;
      }
    }
  }
  uint32_t flags = 0;
  GPA_CUDA(cudaMemcpyAsync(&flags, d_flags.p, 4, cudaMemcpyDeviceToHost, s));
  stream_wait(s);
  for (size_t c = 0; c < C; ++c)
    if (pe[2 * c]) {
      float ms = 0;
      GPA_CUDA(cudaEventElapsedTime(&ms, pe[2 * c], pe[2 * c + 1]));
      pairs_ms += ms;
    }
  const double t1 = wall_ms();
  bs->build_ms[0] = t1 - t0;   // upload (overlapped with the kernels below)

  // ---- global counts, validation (same rules and collectives as bitset_build)
  if ((flags & kFlagNonCanonical) && !(flags & (kFlagBadItem | kFlagBadOffsets))) {
    GPA_CUDA(cudaMemsetAsync(d_hist.p, 0, n_items * 4, s));
    launch_hist_dedup(d_off.p, d_items.p, n_tx, nnz, n_items, d_hist.p, bs->n_sms, s);
  }
  allreduce_max_u32(dist, d_flags.p, 1, s);
  allreduce_sum_u32(dist, d_hist.p, n_items, s);
  if (nr0 >= 2) allreduce_sum_u32(dist, d_r0pairs.p, P0, s);
  bs->item_counts.assign(n_items, 0);
  GPA_CUDA(cudaMemcpyAsync(bs->item_counts.data(), d_hist.p, n_items * 4, cudaMemcpyDeviceToHost, s));
  GPA_CUDA(cudaMemcpyAsync(&flags, d_flags.p, 4, cudaMemcpyDeviceToHost, s));
  stream_wait(s);
  bs->n_tx_global = n_global;
  GPA_REQUIRE(!(flags & kFlagBadOffsets), GPA_ERR_INVALID, "offsets are not non-decreasing%s",
              dist ? " (on some rank)" : "");
  GPA_REQUIRE(!(flags & kFlagBadItem), GPA_ERR_INVALID, "an item id is >= n_items (%u)%s", n_items,
              dist ? " (on some rank)" : "");
  GPA_REQUIRE(bs->n_tx_global < (1ull << 32), GPA_ERR_INVALID, "n_tx must be < 2^32 (32-bit supports)");
  const double t2 = wall_ms();
  bs->build_ms[1] = t2 - t1;

  // ---- rows = L_1 (count >= row_min_count), ascending id
  bs->row_of_item.assign(n_items, -1);
  bool subset = true;
  std::vector<uint32_t> sel;  // position of each L_1 item among the R0 rows
  for (uint32_t i = 0; i < n_items; ++i) {
    if (bs->item_counts[i] >= row_min_count && bs->item_counts[i] > 0) {
      bs->row_of_item[i] = (int32_t)bs->item_of_row.size();
      bs->item_of_row.push_back(i);
      if (r0_of_item[i] < 0) subset = false;
      else sel.push_back((uint32_t)r0_of_item[i]);
    }
  }
  bs->n_rows = (uint32_t)bs->item_of_row.size();
  if (bs->n_rows) {
    if (subset) {
      // L_1 within R0: the R0 bitset IS the static bitset (no row copy); L_1 is listed in bs->l1
      // (R0 row ids) unless it is all of R0
      const uint32_t n1 = bs->n_rows;
      bs->rows = std::move(d_r0rows);
      bs->item_of_row = r0_items;
      bs->row_of_item = r0_of_item;
      bs->n_rows = nr0;
      bs->l1 = sel;
      bs->l1_sub = n1 < nr0;
      DBuf<uint32_t> d_sel;
      d_sel.alloc(n1, s);
      GPA_CUDA(cudaMemcpyAsync(d_sel.p, sel.data(), n1 * 4, cudaMemcpyHostToDevice, s));
      if (n1 >= 2) {
        const uint64_t P = (uint64_t)n1 * (n1 - 1) / 2;
        bs->d_counts.ensure(P, s);
        GPA_CUDA(cudaEventRecord(bs->ev0, s));
        launch_pairs_subset(d_r0pairs.p, nr0, d_sel.p, n1, bs->d_counts.p, bs->n_sms, s);
        GPA_CUDA(cudaEventRecord(bs->ev1, s));
        GPA_CUDA(cudaEventSynchronize(bs->ev1));
        float ms = 0;
        GPA_CUDA(cudaEventElapsedTime(&ms, bs->ev0, bs->ev1));
        *pairs_ready = true;
        if (pair_stats) {
          pair_stats->kernel = pairs_tc ? GPA_KERNEL_PAIRS_TC : GPA_KERNEL_PAIRS;
          pair_stats->launches = pair_launches + 1;
          pair_stats->count_ms = pairs_ms + ms;
          pair_stats->allreduce_ms = 0;
        }
      }
    } else {
      // R0 missed a frequent item: rebuild the L_1 bitset from the device CSR (exact fallback)
      bs->rows.alloc((size_t)bs->n_rows * bs->pitch_words, s);
      DBuf<int32_t> d_map;
      d_map.alloc(n_items, s);
      GPA_CUDA(cudaMemcpyAsync(d_map.p, bs->row_of_item.data(), n_items * 4, cudaMemcpyHostToDevice, s));
      launch_bitset_build(d_off.p, d_items.p, n_tx, nnz, d_map.p, n_items, bs->n_rows, bs->pitch_words, bs->rows.p, 0,
                          n_tx, s);
    }
  }
  stream_wait(s);
  bs->build_ms[2] = wall_ms() - t2;
  if (trace_enabled())
    fprintf(stderr, "[gpa] overlapped ingest: %zu chunks, R0 = %u rows, L1 = %u rows (%s), upload+hist+build+pairs "
            "%.2f ms (pairs kernels %.2f ms), finish %.2f ms; items sent as %u-bit fields and raw (%.1f MB)\n", C, nr0,
            bs->n_rows, subset ? "subset" : "rebuilt", t1 - t0, pairs_ms, wall_ms() - t1, pbits ? pbits : 32,
            packed_bytes / 1e6);
  guard.b = nullptr;
  return bs;
}

}  // namespace gpa
