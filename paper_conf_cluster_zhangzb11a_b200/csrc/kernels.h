// Launch wrappers of the sm_100a kernels (defined in csrc/kernels/*.cu).  All are
// asynchronous on `stream`; all device pointers live on the current device.
#pragma once
#include <cstdint>
#include <functional>
#include <vector>
#include <cuda_runtime.h>

#include "common.h"

namespace gpa {

// ---- generation 1 (P13@338: "test their frequencies by scanning the transaction database")
// Validates the CSR (offsets monotone, items < n_items, canonical order) into *flags and
// accumulates hist[item] += 1 per (transaction, item) incidence.  hist must be zeroed.
// nnz = offsets[n_tx]: a transaction whose offsets leave [0, nnz] is flagged, never read.
void launch_hist_validate(const uint64_t* offsets, const uint32_t* items, uint64_t n_tx, uint64_t nnz,
                          uint32_t n_items, uint32_t* hist, uint32_t* flags, int n_sms, cudaStream_t stream);
// same over transactions [tx_begin, tx_end) (offsets / items are the whole arrays)
// items[j] of a bit-packed upload (bits per item, little-endian 32-bit words) -> out[j] (u32), j < n
void launch_unpack_items(const uint32_t* packed, uint64_t n, uint32_t bits, uint32_t* out, int n_sms,
                         cudaStream_t stream);
void launch_hist_validate_range(const uint64_t* offsets, const uint32_t* items, uint64_t tx_begin, uint64_t tx_end,
                                uint64_t nnz, uint32_t n_items, uint32_t* hist, uint32_t* flags, int n_sms,
                                cudaStream_t stream);
// Same histogram for non-canonical input: an item counts once per transaction (set semantics).
void launch_hist_dedup(const uint64_t* offsets, const uint32_t* items, uint64_t n_tx, uint64_t nnz, uint32_t n_items,
                       uint32_t* hist, int n_sms, cudaStream_t stream);

// ---- static bitset (P18@755): rows[r][t/32] bit t%32 = [item_of_row[r] in t]
// Transactions [tx_begin, tx_end) only (tx_begin a multiple of 512); items >= n_items are skipped.
void launch_bitset_build(const uint64_t* offsets, const uint32_t* items, uint64_t n_tx, uint64_t nnz,
                         const int32_t* row_of_item, uint32_t n_items, uint32_t n_rows, uint64_t pitch_words,
                         uint32_t* rows, uint64_t tx_begin, uint64_t tx_end, cudaStream_t stream);

// Generation-1 counts AND the static bitset of ALL item ids (row = item id, n_items rows of
// pitch_words) in one read of the CSR (bitset.cu scan_build_kernel): hist[i] += popcount of row i
// over this range (set semantics), flags |= kFlagBad*.  hist, flags zeroed by the caller.  Needs
// scan_build_supported(n_items, items) (n_items <= 1,024 and 16-byte aligned items).
bool scan_build_supported(uint32_t n_items, const void* items);
void launch_scan_build(const uint64_t* offsets, const uint32_t* items, uint64_t n_tx, uint64_t nnz, uint32_t n_items,
                       uint64_t pitch_words, uint32_t* rows, uint32_t* hist, uint32_t* flags, cudaStream_t stream);
// In place: row r <- row sel[r] for r in [r0, n_sel) (sel ascending, sel[r] >= r).
void launch_compact_rows(uint32_t* rows, const uint32_t* sel, uint32_t r0, uint32_t n_sel, uint64_t pitch_words,
                         int n_sms, cudaStream_t stream);

// ---- support counting (complete intersection, P18@394-2515)
// Paper design: one CTA per candidate, AND of all k rows, popc, block reduction.
void launch_count_v0(const uint32_t* rows, uint64_t pitch_words, const uint32_t* cand_rows, uint32_t k,
                     uint64_t M, uint32_t* counts, cudaStream_t stream);

// Prefix-staged streaming: groups share a (k-1)-prefix; counts must be zeroed (atomic adds).
struct PrefixTask {
  uint32_t group;   // prefix group
  uint32_t first;   // index of the first sibling (global candidate index)
  uint32_t n;       // siblings in this task (<= kPrefixMaxSiblings)
  uint32_t pad;
};
constexpr uint32_t kPrefixMaxSiblings = 32;
// returns the number of CTAs launched
uint64_t launch_count_prefix(const uint32_t* rows, uint64_t pitch_words, const uint32_t* prefix_rows, uint32_t km1,
                             const uint32_t* ext_rows, const PrefixTask* tasks, uint32_t n_tasks, uint32_t* counts,
                             cudaStream_t stream);

// Transaction-tiled trie walk for generations k in [2, kTrieMaxK] (count_trie.cu).  Candidates
// (lexicographic) are cut into blocks of <= kTrieMaxCand candidates touching <= kTrieMaxRows rows.
constexpr uint32_t kTrieMaxK = 16;
constexpr uint32_t kTrieMaxRows = 64;    // k = 2: 4 words per lane (128-word stripes), <= 64 rows / block
constexpr uint32_t kTrieWideRows = 32;   // k >= 3: 8 words per lane (256-word stripes), <= 32 rows / block
constexpr uint32_t kTrieMaxCand = 256;
struct TrieBlock {
  uint32_t cand_begin;   // first candidate (global index)
  uint32_t n_cand;       // <= kTrieMaxCand
  uint32_t row_begin;    // into block_rows
  uint32_t n_rows;       // <= trie_max_rows(k)
};
inline bool trie_wide(uint32_t k) { return k >= 3; }
inline uint32_t trie_max_rows(uint32_t k) { return trie_wide(k) ? kTrieWideRows : kTrieMaxRows; }
inline uint32_t trie_stripe_words(uint32_t k) { return trie_wide(k) ? 256 : 128; }
// cand_lrows[c]: byte d = block-local row of item d; cand_lcp[c]: items shared with candidate c-1
// (0 for the first candidate of every warp chunk: a block's n candidates are split into chunks of
// ceil(n / 8)).  counts must be zeroed.
uint64_t launch_count_trie(uint32_t k, const uint32_t* rows, uint64_t pitch_words, const TrieBlock* blocks,
                           const uint32_t* block_rows, const uint4* cand_lrows, const uint8_t* cand_lcp,
                           uint32_t n_blocks, uint32_t max_rows, uint32_t n_parts, uint32_t* counts,
                           cudaStream_t stream);

// k = 2 TMA-tiled kernel: all pairs (a < b) of the n_rows rows; counts[pair_index] must be zeroed.
// tmap: opaque 128-byte CUtensorMap built by make_pairs_tensor_map.
bool make_pairs_tensor_map(void* tmap128, const uint32_t* rows, uint32_t n_rows, uint64_t pitch_words);
// Words [word_begin, word_end) of the rows (multiples of 32); counts accumulate (atomic adds).
uint64_t launch_count_pairs(const void* tmap128, uint32_t n_rows, uint64_t word_begin, uint64_t word_end,
                            uint32_t* counts, int n_sms, cudaStream_t stream);
// k = 2 on the tensor cores (count_pairs_tc.cu): C = B B^T over words [word_begin, word_end)
// (multiples of 4) as a tcgen05 kind::i8 GEMM of the bit-expanded rows; counts accumulate.
uint64_t launch_count_pairs_tc(const uint32_t* rows, uint64_t pitch_words, uint32_t n_rows, uint64_t word_begin,
                               uint64_t word_end, uint32_t* counts, int n_sms, cudaStream_t stream);
inline bool pairs_kernel_k2(uint32_t kernel) {
  return kernel == GPA_KERNEL_AUTO || kernel == GPA_KERNEL_PAIRS || kernel == GPA_KERNEL_PAIRS_TC ||
         kernel == GPA_KERNEL_PROJ;
}
// counts_sub[pair_index(a, b, n_sub)] = counts_all[pair_index(sel[a], sel[b], n_all)] (sel ascending)
void launch_pairs_subset(const uint32_t* counts_all, uint32_t n_all, const uint32_t* sel, uint32_t n_sub,
                         uint32_t* counts_sub, int n_sms, cudaStream_t stream);
// rows_sub[r] = rows_all[sel[r]] (whole rows of pitch_words words)
void launch_gather_rows(const uint32_t* rows_all, const uint32_t* sel, uint32_t n_sub, uint64_t pitch_words,
                        uint32_t* rows_sub, int n_sms, cudaStream_t stream);

// ---- device-side level transition (candgen.cu)
// Status words of the single-launch scans (scan.cu): per tile a flag (epoch << 2 | 1 aggregate /
// 2 inclusive) and the two values; the epoch advances per scan, so nothing is cleared between
// scans.  One per stream at a time (scans on one state must be stream-ordered).
struct ScanState {
  PBuf<uint32_t> flags;
  PBuf<uint64_t> agg, inc;
  uint32_t epoch = 0;
};
// fused scans (scan_dev.cuh): tiles of a scan of n values (items per thread), and the epoch of
// the next scan on st
uint32_t scan_tiles(uint32_t n, uint32_t items = 8);
uint32_t scan_epoch(ScanState& st, uint32_t tiles, cudaStream_t s);
void scan_excl_u32(const uint32_t* in, uint32_t* out, uint32_t n, uint32_t* tot, ScanState& st, cudaStream_t s);
void scan_excl_u32(const uint32_t* in, uint32_t* out, uint32_t n, uint64_t* tot, ScanState& st, cudaStream_t s);
void scan_excl_u64(const uint64_t* in, uint64_t* out, uint32_t n, uint64_t* tot, ScanState& st, cudaStream_t s);
// the two above in one launch (independent inputs)
void scan_excl_dual(const uint32_t* in1, uint32_t* out1, uint32_t n1, uint64_t* tot1, const uint64_t* in2,
                    uint64_t* out2, uint32_t n2, uint64_t* tot2, ScanState& st, cudaStream_t s);
// (cnt << 32 | cnt != 0) scanned as one: off = exclusive sums of cnt, idx = exclusive count of the
// non-zero cnt, tot2 = {sum, non-zero count}
void scan_excl_split(const uint32_t* cnt, uint32_t* off, uint32_t* idx, uint32_t n, uint32_t* tot2, ScanState& st,
                     cudaStream_t s);

// Its scan status words persist per thread and device (scan_state()): they are cudaMalloc'd
// (PBuf), and a per-call ScanState would allocate -- and on growth cudaFree, which synchronises
// the device -- inside every mining call.
ScanState& scan_state(int device);
struct DeviceScratch {
  explicit DeviceScratch(int device) : scan(scan_state(device)) {}
  DBuf<uint32_t> a, b, c, d, e, f, g, h, i;
  uint32_t hash_cap = 0;   // slots of the join's hash set (i), filled by the scatter of L (threshold)
  // the run structure stage 1 used (its own run scan, or the class scan of the projected lists: a
  // class of L -- entries with one left parent -- IS a run of L), for stage 2
  const uint32_t *rflags = nullptr, *rex = nullptr, *rbound = nullptr;
  uint32_t hash_n = 0;     // the level size (upper bound) that set was built for
  ScanState& scan;
  uint32_t* u32a(size_t n, cudaStream_t s) { a.ensure(n ? n : 1, s); return a.p; }
  uint32_t* u32b(size_t n, cudaStream_t s) { b.ensure(n ? n : 1, s); return b.p; }
  uint32_t* u32c(size_t n, cudaStream_t s) { c.ensure(n ? n : 1, s); return c.p; }
  uint32_t* u32d(size_t n, cudaStream_t s) { d.ensure(n ? n : 1, s); return d.p; }
  uint32_t* u32e(size_t n, cudaStream_t s) { e.ensure(n ? n : 1, s); return e.p; }
  uint32_t* u32f(size_t n, cudaStream_t s) { f.ensure(n ? n : 1, s); return f.p; }
  uint32_t* u32g(size_t n, cudaStream_t s) { g.ensure(n ? n : 1, s); return g.p; }
  uint32_t* u32h(size_t n, cudaStream_t s) { h.ensure(n ? n : 1, s); return h.p; }
  uint32_t* u32i(size_t n, cudaStream_t s) { i.ensure(n ? n : 1, s); return i.p; }
  // one generation's sizes, read by the host in ONE copy: [0] |C_k|, [1] groups, [2..5] the lists'
  // totals (u64 x 2: build items, words), [6..9] class-table counters (classes, max lane words,
  // u64 compressed words), [10] |L_{k-1}|
  DBuf<uint32_t> blk;
  uint32_t* size_block(cudaStream_t s) { blk.ensure(16, s); return blk.p; }
  // the join's per-member survivor masks (stage 1 -> stage 2, lvl::join_warp)
  DBuf<unsigned long long> surv;
  unsigned long long* surv64(size_t n, cudaStream_t s) { surv.ensure(n ? n : 1, s); return surv.p; }
};
// L_k on the device: n rows of k row ids (lexicographic) and their supports
// par_a[p] / par_b[p]: index in L_{k-1} of the entry's left parent (its first k-1 items) and
// right parent (first k-2 items + last item); for k = 2 the two row ids.  Used by the projected
// lists of proj.cu.
// Device-sized level (n_dev != nullptr): |L| is only on the device (*n_dev, = count.p) until the
// next synchronisation, the arrays hold n_max (>= |L|) entries; the level-transition kernels read
// the count from the device and run over the upper bound.
struct DeviceLevel {
  uint32_t k = 0, n = 0;
  DBuf<uint32_t> rows, sup, par_a, par_b, count;
  const uint32_t* n_dev = nullptr;
  uint32_t n_max = 0;
};
// C_k on the device, grouped by (k-1)-prefix: prefix[G][k-1], ext_off[G+1], ext[M]
// gpar[g] = index in L_{k-1} of group g's prefix (the left parent), eidx[m] = index in L_{k-1} of
// candidate m's right parent (prefix without its last item, plus ext[m]).
struct DeviceBatch {
  uint32_t k = 0, M = 0, G = 0;
  DBuf<uint32_t> prefix, ext_off, ext, gpar, eidx;
};
// L_k = candidates of C_k with count >= theta, in order (k = 2: all pairs of n_rows L_1 entries in
// pair_index order, mapped to bitset rows through sel when non-null; k >= 3: the grouped batch
// prefix/ext_off/ext).  Returns |L_k| (synchronises).  With gpar / eidx (k >= 3) or always for
// k = 2, also out.par_a / out.par_b.
uint32_t device_threshold(const uint32_t* counts, uint32_t M, uint32_t theta, uint32_t k, uint32_t n_rows,
                          const uint32_t* sel, const uint32_t* prefix, const uint32_t* ext_off, const uint32_t* ext,
                          uint32_t G, const uint32_t* gpar, const uint32_t* eidx,
                          DeviceLevel& out, DeviceScratch& scratch, int n_sms, cudaStream_t s);
// The same without a synchronisation: out becomes device-sized (n_dev = &|L_k|, n_max = M).  With
// items / sup_out (>= M k / M words) the scatter also writes L_k's original item ids (ior: bitset
// row -> item id) and supports for the result.
void device_threshold_async(const uint32_t* counts, uint32_t M, uint32_t theta, uint32_t k, uint32_t n_rows,
                            const uint32_t* sel, const uint32_t* prefix, const uint32_t* ext_off, const uint32_t* ext,
                            uint32_t G, const uint32_t* gpar, const uint32_t* eidx,
                            DeviceLevel& out, DeviceScratch& scratch, int n_sms, cudaStream_t s,
                            const uint32_t* ior = nullptr, uint32_t* items = nullptr, uint32_t* sup_out = nullptr);

// ---- association rules (rules.cu): F as n itemsets in canonical order (items at
// items + item_off[i], len[i] items, support sup[i]); the rules A => X \ A of the itemsets x0 .. n-1
// (those with |X| >= 2) with supp(X) * den >= num * supp(A), as (X index, antecedent mask, supp(A))
// in (X, mask) order.  num, den < 2^32.  The rules land in host_alloc(n_rules): 3 x n_rules words
// (X indices, masks, supports of A).  Returns n_rules.  Synchronises.
uint64_t device_rules(const uint32_t* items, const uint64_t* item_off, const uint32_t* len, const uint32_t* sup,
                      uint32_t n, uint32_t x0, uint64_t num, uint64_t den, int n_sms, cudaStream_t s,
                      const std::function<uint32_t*(uint64_t)>& host_alloc);

// ---- projected vertical lists (proj.cu; "equivalent class clustering", P13@2288-2486)
// For every entry j of a level L (n entries with parents par_a / par_b): the bits of its last
// item's row restricted to the transactions of its class (the entries with the same par_a), in
// the class' position order.  Entries of single-member classes (no candidates) get no vector.
// Buffers are persistent and grow-only (PBuf): one DeviceProj pair per thread and device lives
// across generations and mining calls (proj_lists()).
struct DeviceProj {
  uint32_t n = 0;
  PBuf<uint64_t> off;     // n: word offset of entry j's vector in data
  PBuf<uint32_t> nw;      // n: words of entry j's vector (multiple of 32; 0 = none)
  PBuf<uint32_t> data;
  uint64_t words = 0;
  uint32_t max_lw = 0;    // longest lane stream (words) of any class
  uint64_t in_words = 0;  // mask words x members compressed to build these lists (algorithmic work)
};
// The calling thread's two DeviceProj for `device` (previous / current generation).
DeviceProj* proj_lists(int device);
// Vectors of L = L_{k-1} from the previous level's vectors (prev = those of L_{k-2}) or, for
// L = L_2 (prev == nullptr), from the bitset rows.  Synchronises once (sizes).  Returns false
// when the vectors do not fit (device memory / 32-bit totals): use complete intersection.
bool proj_build(uint32_t n, const uint32_t* par_a, const uint32_t* par_b, const DeviceProj* prev,
                const uint32_t* rows, uint64_t pitch_words, uint32_t n_rows, DeviceProj& out, DeviceScratch& scratch,
                int n_sms, cudaStream_t s, cudaEvent_t ev_build = nullptr);
// The same in two stages around one host read of the sizes: begin enqueues the class tables and
// leaves the totals on the device (pp.d_tot: u64[2] = pext items, list words; pp.d_small: u32[4]),
// finish (given those values) sizes the lists and launches the list build.
struct ProjPending {
  uint32_t n = 0, cmax = 0, nseg = 0, n_pairs = 0;
  int device = 0;
  const uint32_t *par_a = nullptr, *par_b = nullptr, *rows = nullptr;
  const DeviceProj* prev = nullptr;
  uint64_t pitch = 0;
  const uint64_t* d_tot = nullptr;
  const uint32_t* d_small = nullptr;
  const uint32_t *flag = nullptr, *ex = nullptr, *bound = nullptr;   // the class scan (null: not run)
};
// begin returns false (nothing enqueued) when the lists cannot be addressed (bitset >= 2^32 words,
// too many classes): use complete intersection.
// n_dev: L is device-sized (n = its host upper bound, the count at *n_dev); set pp.n to the count
// before proj_build_finish.
// d_block (optional): the generation's size block (DeviceScratch::size_block): the totals and the
// class-table counters are written to words 2..9 of it instead of the workspace's own
// pre / fork (optional): the class scan runs on `pre`, then s waits for `fork` recorded after it (the
// class scan's flag / ex / bound arrays -- pp.flag, pp.ex, pp.bound -- are L's runs as well)
bool proj_build_begin(uint32_t n, const uint32_t* par_a, const uint32_t* par_b, const DeviceProj* prev,
                      const uint32_t* rows, uint64_t pitch_words, uint32_t n_rows, DeviceScratch& scratch, int n_sms,
                      cudaStream_t s, ProjPending& pp, const uint32_t* n_dev = nullptr, uint32_t* d_block = nullptr,
                      cudaStream_t pre = nullptr, cudaEvent_t fork = nullptr);
bool proj_build_finish(const ProjPending& pp, const uint64_t T[2], const uint32_t sm[4], DeviceProj& out, int n_sms,
                       cudaStream_t s, cudaEvent_t ev_build);
// counts[m] += popc(V_gpar[g] & V_eidx[m]) for every candidate m of group g (counts zeroed by the caller,
// unless count_proj_stores_all(P): the warp-per-group variant of short lists stores every count)
bool count_proj_stores_all(const DeviceProj& P);
void launch_count_proj(const DeviceProj& P, const uint32_t* gpar, const uint32_t* ext_off, const uint32_t* eidx,
                       uint32_t G, uint32_t* counts, cudaStream_t s);
// items[i] = item_of_row[rows[i]] (row ids -> original item ids) for i < n, or for i < *n_dev * k
// when n_dev is given (n then an upper bound)
void device_map_items(const uint32_t* rows, uint64_t n, const uint32_t* item_of_row, uint32_t* items, int n_sms,
                      cudaStream_t s, const uint32_t* n_dev = nullptr, uint32_t k = 1,
                      const uint32_t* sup_in = nullptr, uint32_t* sup_out = nullptr);
// exclusive scan of n u32 (CUB); the total is written to *tot (device) when tot != nullptr
void device_exclusive_scan(const uint32_t* in, uint32_t* out, uint32_t n, uint32_t* tot, DeviceScratch& scratch,
                           cudaStream_t s);
// C_{k+1} = join + prune of L (k >= 2), grouped by k-prefix (synchronises for the sizes).
void device_candgen(const DeviceLevel& L, DeviceBatch& out, DeviceScratch& scratch, int n_sms, cudaStream_t s);
// The same in two stages around one host read of the sizes (so that another stage-1 -- the
// projected lists' class tables -- can share the synchronisation): begin leaves (M, G) at
// *d_sizes on the device; finish sizes the batch on s and runs the emitting join on `run`
// (waiting for s through ev when run != s).  begin returns false when |L| < 2 (no candidates).
// runs (optional): flags / exclusive counts / bounds of L's runs already on the device (the class
// scan of proj_build_begin, ordered before on s): no run-detection scan of its own
bool device_candgen_begin(const DeviceLevel& L, DeviceBatch& out, DeviceScratch& scratch, int n_sms, cudaStream_t s,
                          const uint32_t** d_sizes, const uint32_t* run_flags = nullptr,
                          const uint32_t* run_ex = nullptr, const uint32_t* run_bound = nullptr);
void device_candgen_finish(const DeviceLevel& L, DeviceBatch& out, DeviceScratch& scratch, int n_sms, cudaStream_t s,
                           uint32_t M, uint32_t G, cudaStream_t run, cudaEvent_t ev);

// ---- the whole level loop in one cooperative launch for small problems (mine_fused.cu)
constexpr uint32_t kFusedMaxRows = 1024;                      // |L_1| (a 32-word tile of every row: 128 KB)
constexpr uint64_t kFusedMaxBitsetBytes = 48ull << 20;        // L_1 rows (L2-resident)
bool fused_eligible(uint32_t n1, uint64_t pitch_words);
struct FusedOut {
  struct Level {
    uint32_t k = 0, M = 0, F = 0, G = 0;
    uint64_t freq_word = 0, freq_entry = 0, cand_word = 0, cand_entry = 0;   // offsets into the arrays below
  };
  std::vector<Level> levels;               // generations 2 .. last
  // L_k item ids (F x k per generation) and supports, in order: copied from the device into one
  // page-locked block from pinned_alloc (bytes in, rounded size out)
  std::function<void*(size_t&)> pinned_alloc;
  const uint32_t* items = nullptr;
  const uint32_t* sup = nullptr;
  std::vector<uint32_t> cand_items, cand_counts;   // keep: every C_k (M x k) and its counts
};
// Levels k >= 2 of gpa_mine over the L_1 rows (n1 entries; d_sel: entry -> bitset row or nullptr;
// d_ior: bitset row -> item id).  false: a capacity was exceeded (nothing usable in out).
// c2_counts: generation 2's counts (pair order over the n1 entries) already on the device, or
// nullptr to count them in the fused loop.
bool mine_fused(const uint32_t* rows, uint64_t pitch_words, uint64_t n_tx, uint32_t n1, const uint32_t* d_sel,
                const uint32_t* d_ior, uint32_t theta, uint32_t max_k, bool keep, int n_sms, cudaStream_t s,
                FusedOut& out, const uint32_t* c2_counts = nullptr);
constexpr uint32_t kFusedPairsTcRows = 128;   // above this |L_1|, generation 2 runs on the tensor cores first

// ---- device-side work planning (plan.cu)
constexpr uint32_t kPlanMaxRows = 65536;   // row bitmap of the planning kernels (8 KB of shared memory)
void launch_cand_group(const uint32_t* ext_off, uint32_t G, uint32_t* cand_group, int n_sms, cudaStream_t s);
// R[w] = distinct rows of the candidates [windows[w].x, windows[w].x + windows[w].y)
void launch_window_rows(const uint32_t* prefix, const uint32_t* ext, const uint32_t* cand_group, uint32_t k,
                        uint32_t n_rows, const uint2* windows, uint32_t n_windows, uint32_t* R, cudaStream_t s);
// greedy partition of each window of `window` candidates into blocks of <= rmax distinct rows:
// recs[w * window + i] = {first candidate, count, rows}, n_recs[w] = number of blocks of window w
void launch_window_greedy(const uint32_t* prefix, const uint32_t* ext, const uint32_t* cand_group, uint32_t k,
                          uint32_t n_rows, uint32_t M, uint32_t window, uint32_t rmax, uint3* recs, uint32_t* n_recs,
                          cudaStream_t s);
// blocks[off[w] + i] = record i of window w (row_begin left 0), rows[] = their row counts,
// stats[0] = max(rows) (must be zeroed); then row_begin[b] = row_off[b]
void launch_compact_blocks(const uint3* recs, const uint32_t* n_recs, const uint32_t* off, uint32_t n_win,
                           uint32_t window, TrieBlock* blocks, uint32_t* rows, uint32_t* stats, cudaStream_t s);
void launch_row_begin(const uint32_t* row_off, uint32_t n_blocks, TrieBlock* blocks, int n_sms, cudaStream_t s);
// per block (row_begin set, n_rows an upper bound): row list, exact n_rows, candidates' local row
// bytes and lcp (count_trie's format)
void launch_build_blocks(const uint32_t* prefix, const uint32_t* ext, const uint32_t* cand_group, uint32_t k,
                         uint32_t n_rows, TrieBlock* blocks, uint32_t n_blocks, uint32_t* trows, uint4* lrows,
                         uint8_t* lcp, cudaStream_t s);
// write == false: n_tasks[g] = ceil(|group g| / 32); write == true: tasks at task_off
void launch_prefix_tasks(const uint32_t* ext_off, uint32_t G, uint32_t* n_tasks, const uint32_t* task_off,
                         PrefixTask* tasks, int n_sms, cudaStream_t s, bool write);

}  // namespace gpa
