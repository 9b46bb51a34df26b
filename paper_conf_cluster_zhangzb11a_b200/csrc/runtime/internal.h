// Runtime-internal declarations (handles, device buffers, counting engine).
#pragma once
#include <nvtx3/nvToolsExt.h>
#include <cstdint>
#include <cstring>
#include <string>
#include <utility>
#include <vector>
#include <new>
#include <exception>

#include <cuda_runtime.h>
#include <nccl.h>

#include "../common.h"
#include "../kernels.h"

struct gpa_dist {
  ncclComm_t comm = nullptr;           // NCCL transport (gpa_dist_create)
  gpa_host_allreduce_fn host_fn = nullptr;   // host-staged transport (gpa_dist_create_host)
  void* host_ctx = nullptr;
  int rank = 0, world = 1, device = 0;
  bool failed = false;
  double timeout_s = 600.0;
  std::vector<uint64_t> log;           // (op << 60) | (dtype << 56) | n of every collective, in order
  void* stage = nullptr;               // pinned staging of the host transport
  size_t stage_bytes = 0;
};

namespace gpa {
// NVTX range (header-only NVTX v3: a no-op unless a profiler is attached): phases of gpa_mine show
// up by name in Nsight Systems / ncu --nvtx
struct NvtxRange {
  explicit NvtxRange(const char* name) { nvtxRangePushA(name); }
  NvtxRange(const NvtxRange&) = delete;
  NvtxRange& operator=(const NvtxRange&) = delete;
  ~NvtxRange() { nvtxRangePop(); }
};

struct DeviceInfo {
  int device;
  int n_sms;
};
DeviceInfo use_device(int requested);   // cudaSetDevice + one-time pool setup

// Collective helpers (no-ops without dist; NCCL or the host-staged transport)
void dist_check(const gpa_dist* d);
void allreduce_sum_u32(const gpa_dist* d, uint32_t* buf, size_t n, cudaStream_t s);
void allreduce_sum_u64(const gpa_dist* d, uint64_t* buf, size_t n, cudaStream_t s);
void allreduce_max_u32(const gpa_dist* d, uint32_t* buf, size_t n, cudaStream_t s);
// Element-wise max over ranks of a few host values (one small collective on a library stream of
// the dist's device; identity without dist).  Every path decision that changes the collective
// sequence goes through it so that all ranks take the same branch.
void dist_agree_max(const gpa_dist* d, uint32_t* vals, size_t n);
// While alive, waits on streams (stream_wait) of this thread poll d's NCCL communicator for
// asynchronous errors and time out after d->timeout_s.
struct DistScope {
  const gpa_dist* prev;
  explicit DistScope(const gpa_dist* d);
  ~DistScope();
};

// Candidate batch grouped by (k-1)-prefix, in ROW ids.  Candidates are prefix + ext[j] for
// j in [ext_off[g], ext_off[g+1]); global candidate index = position in ext.
struct GroupedBatch {
  uint32_t k = 0;
  std::vector<uint32_t> prefix;    // G * (k-1)
  std::vector<uint64_t> ext_off;   // G + 1
  std::vector<uint32_t> ext;       // M
  uint64_t groups() const { return ext_off.empty() ? 0 : ext_off.size() - 1; }
  uint64_t size() const { return ext.size(); }
};

// Join + prune of L_{k-1} (n x (k-1) row ids, lexicographic, distinct) into C_k grouped by
// (k-1)-prefix; candidates come out in lexicographic order.
GroupedBatch candgen_join_prune(const std::vector<uint32_t>& L, uint64_t n, uint32_t km1);

// Work plan of the trie kernel for a grouped batch (host side; see count_trie.cu): blocks of
// <= kTrieMaxCand lexicographically consecutive candidates touching <= trie_max_rows(k) rows, the
// block-local row byte of every item of every candidate, and the shared-prefix length with the
// previous candidate (0 at the start of every warp chunk of ceil(n_cand / 8) candidates).
struct TriePlan {
  std::vector<TrieBlock> blocks;
  std::vector<uint32_t> rows;     // global row ids, concatenated per block
  std::vector<uint4> lrows;       // M entries: byte d = local row of item d
  std::vector<uint8_t> lcp;       // M entries
  uint32_t max_rows = 0;
};
TriePlan plan_trie(const GroupedBatch& b, uint32_t n_rows);

const char* last_error_cstr();

// Host tracing (SURVEY.md §5 "Tracing"): GPA_TRACE=1 prints one line per mining phase / level
// with host wall-clock splits to stderr.
bool trace_enabled();
double wall_ms();

// Run f() and translate exceptions into a gpa_status + thread-local message (no exception
// crosses the C ABI).
template <class F>
gpa_status guard(F&& f) {
  try {
    f();
    return GPA_OK;
  } catch (const Error& e) {
    set_last_error(e.status, e.msg);
    return e.status;
  } catch (const std::bad_alloc&) {
    set_last_error(GPA_ERR_OOM, "host allocation failed");
    return GPA_ERR_OOM;
  } catch (const std::exception& e) {
    set_last_error(GPA_ERR_INVALID, std::string("internal error: ") + e.what());
    return GPA_ERR_INVALID;
  } catch (...) {
    set_last_error(GPA_ERR_INVALID, "internal error");
    return GPA_ERR_INVALID;
  }
}

struct CountStats {
  uint32_t kernel = 0;
  uint32_t launches = 0;
  double count_ms = 0;
  double allreduce_ms = 0;
  // optional caller-owned events: with them the counting functions do not synchronise; the
  // caller reads count_ms / allreduce_ms from (e0, e1) / (e1, e2) later
  cudaEvent_t e0 = nullptr, e1 = nullptr, e2 = nullptr;
  cudaEvent_t ep = nullptr, eb = nullptr;  // GPA_KERNEL_PROJ: the list-building kernel (ep .. eb)
  uint64_t build_words = 0;
  uint64_t build_bytes = 0, count_bytes = 0;   // GPA_KERNEL_PROJ: algorithmic bytes (gpa_level_stats)
};

// A stream + three timing events, recycled across bitsets (stream / event creation costs ~10 us
// each, and the mining entry points create a bitset per call).  acquire() hands out a free bundle of
// the device or creates one; release() returns it (its stream idle).
struct StreamBundle {
  int device = 0;
  cudaStream_t s = nullptr;
  cudaEvent_t ev[3] = {nullptr, nullptr, nullptr};
};
StreamBundle* acquire_bundle(int device);
void release_bundle(StreamBundle* b);

}  // namespace gpa

struct gpa_bitset {
  int device = 0;
  int n_sms = 148;
  cudaStream_t stream = nullptr;
  gpa::StreamBundle* bundle = nullptr;   // own stream (when opt.stream is null) and ev0..ev2
  const gpa_dist* dist = nullptr;
  gpa_options opt{};
  uint64_t n_tx_local = 0, n_tx_global = 0;
  uint32_t n_items = 0, n_rows = 0;
  uint64_t pitch_words = 0;
  gpa::DBuf<uint32_t> rows;
  std::vector<uint32_t> item_counts;   // global, n_items
  std::vector<uint32_t> item_of_row;   // n_rows, ascending
  std::vector<int32_t> row_of_item;    // n_items, -1 if no row
  // gpa_mine: the rows of L_1 when the bitset holds more rows than L_1 (all item ids after the
  // one-pass build, the chunk-0 estimate R0 after the overlapped ingest): ascending row ids; empty =
  // every row is in L_1.  Generation 2 counts pairs of these rows; L_k holds bitset row ids.
  std::vector<uint32_t> l1;
  bool l1_sub = false;                 // l1 is in use (possibly empty: nothing frequent)
  gpa::DBuf<uint32_t> d_l1, d_pairs_all;
  alignas(64) unsigned char tmap[128];
  bool tmap_ready = false;
  // counting workspace (grow-only)
  gpa::DBuf<uint32_t> d_counts, d_prefix, d_ext, d_flat;
  gpa::DBuf<gpa::PrefixTask> d_tasks;
  gpa::DBuf<gpa::TrieBlock> d_tblocks;
  gpa::DBuf<uint32_t> d_trows;
  gpa::DBuf<uint4> d_lrows;
  gpa::DBuf<uint8_t> d_lcp;
  gpa::DBuf<uint32_t> d_cgroup;      // candidate -> group (device planning)
  cudaEvent_t ev0 = nullptr, ev1 = nullptr, ev2 = nullptr;
  double build_ms[3] = {0, 0, 0};      // upload, histogram, bitset
};

namespace gpa {
// Build the static bitset (histogram, rows, bitset) -- shared by gpa_bitset_create / gpa_mine.
// prechecked: the caller already ran agree_input for db (gpa_mine)
// keep_all_rows (gpa_mine): with the one-pass build, keep the rows of every item id and list
// L_1 in bs->l1 instead of compacting the rows.
gpa_bitset* bitset_build(const gpa_tx_csr* db, uint64_t row_min_count, const gpa_dist* dist, const gpa_options* opt,
                         bool prechecked = false, bool keep_all_rows = false);
// number of L_1 rows (bs->l1, or every row)
inline uint32_t l1_size(const gpa_bitset* bs) { return bs->l1_sub ? (uint32_t)bs->l1.size() : bs->n_rows; }
void bitset_free(gpa_bitset* bs);
// Host input, end to end: upload in transaction chunks overlapped with histogram, bitset build and
// generation-2 pair counting (runtime/ingest.cpp).  *pairs_ready: bs->d_counts holds the L_1 pair
// counts (pair_stats describes the kernels).
bool ingest_overlap_eligible(const gpa_tx_csr* db);
// transaction boundaries of the overlapped ingest's upload chunks: cut[0] = 0 .. cut.back() = n_tx
std::vector<uint64_t> ingest_cuts(uint64_t n_tx);
// Host-side input checks every rank runs BEFORE its first collective, agreed across ranks with one
// small max all-reduce (a rank-local rejection must not strand the others inside a collective):
// throws GPA_ERR_INVALID on every rank alike if any rank's input is malformed or the ranks disagree
// on n_items.  Returns whether EVERY rank can take the overlapped ingest (want_overlap and
// ingest_overlap_eligible on all ranks): a collective decision, so all ranks issue the same
// collective sequence.
bool agree_input(const gpa_tx_csr* db, const gpa_dist* dist, bool want_overlap);
gpa_bitset* bitset_build_overlapped(const gpa_tx_csr* db, uint64_t row_min_count, const gpa_dist* dist,
                                    const gpa_options* opt, bool* pairs_ready, struct CountStats* pair_stats);
// Count a grouped batch into bs->d_counts (device, M entries, summed over ranks).
void count_grouped(gpa_bitset* bs, const GroupedBatch& b, uint32_t kernel, CountStats* st);
// Count a device-resident grouped batch with device-side planning (trie blocks / prefix tasks);
// returns false when it cannot (kernel v0, too many rows) and the host path must be used.
bool count_device_batch(gpa_bitset* bs, DeviceBatch& B, uint32_t kernel, DeviceScratch& scratch, CountStats* st);
// After a counting launch: end event, all-reduce of the M counts (dist), and the timing (no sync
// when st carries caller-owned events).
void finish_counts(gpa_bitset* bs, size_t M, CountStats* st);
// Count all pairs of L_1 rows (bs->l1, or every row; lexicographic pair order) into bs->d_counts
// (n(n-1)/2 entries, n = l1_size).
void count_all_pairs(gpa_bitset* bs, uint32_t kernel, CountStats* st);
}  // namespace gpa
