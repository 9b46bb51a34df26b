/*
 * gpapriori.h -- C ABI of the B200-native GPApriori support-counting library
 *                (libgpapriori.so, built from paper_conf_cluster_zhangzb11a_b200/csrc).
 *
 * The paper (Zhang, Zhang & Bakos, "GPApriori: GPU-Accelerated Frequent Itemset Mining",
 * IEEE Cluster 2011; /root/reference/PAPER.md, cited as P<line>@<char offset>) states the
 * problem as: transactions are sets of items (P3@441); the support ratio of an itemset is
 * the number of transactions containing it divided by the number of transactions (P3@613 -
 * P4@0); given a minimum support ratio, return all frequent itemsets (P4@111).  Its GPU
 * method keeps one "static bitset" row per first-generation (frequent) item in GPU memory
 * (P2@270, P18@755), aligned to 64 bytes (P18@1685), and computes the support of a
 * k-candidate by "complete intersection": popcount of the AND of its k rows (P18@394-1300,
 * Fig. 4 P18@863).  The three entry-point families below are that statement of the
 * problem: build the bitset from a transaction list (gpa_bitset_create), count the
 * supports of a candidate batch (gpa_count), and run level-wise mining with join + prune
 * candidate generation (gpa_mine).
 *
 * Conventions (all entry points):
 *  - extern "C", plain pointers and sizes only.  Every call returns gpa_status; on a
 *    non-OK status a thread-local message is available from gpa_last_error().  No C++
 *    exception, abort() or exit() crosses this boundary.
 *  - Inputs are BORROWED for the duration of the call and copied before return; the caller
 *    may free them afterwards.  Handles (gpa_bitset, gpa_result, gpa_dist) are library-owned
 *    and released with the matching *_destroy; destroying NULL is a no-op returning GPA_OK.
 *  - Output arrays passed by the caller (counts_out, ...) are caller-allocated HOST memory
 *    unless the name says _dev.  Pointers returned through gpa_result_* stay valid until
 *    gpa_result_destroy().
 *  - Item ids are uint32 < n_items.  Supports are uint32 (exact; N < 2^32, the paper's
 *    32-bit per-thread counts P18@1792).  Thresholds compare with >= (Q1).
 *  - Thread-compatible: one handle is used by one host thread at a time.
 *  - Errors: GPA_ERR_INVALID  malformed input (non-monotone offsets, offsets[0] != 0, an item
 *                             >= n_items, a candidate row not strictly increasing, k == 0,
 *                             k > GPA_MAX_K, size overflow, NULL pointer);
 *            GPA_ERR_RANGE    a candidate item owns no bitset row (its count < row_min_count);
 *            GPA_ERR_OOM      device or host allocation failed;
 *            GPA_ERR_CUDA / GPA_ERR_NCCL  the underlying error string is in gpa_last_error();
 *            GPA_ERR_STATE    a handle used after a failed collective, or a device mismatch.
 *    A failed call leaves its output arguments unspecified and allocates nothing the caller
 *    must free.
 *  - No CPU fallback: every counting step runs in this library's sm_100a kernels.
 */
#ifndef GPAPRIORI_H
#define GPAPRIORI_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define GPA_MAX_K 64u          /* longest candidate accepted by gpa_count / mined by gpa_mine */

typedef enum {
  GPA_OK = 0,
  GPA_ERR_INVALID = 1,
  GPA_ERR_RANGE = 2,
  GPA_ERR_OOM = 3,
  GPA_ERR_CUDA = 4,
  GPA_ERR_NCCL = 5,
  GPA_ERR_STATE = 6
} gpa_status;

/* Message of the last non-OK status returned on this host thread; never NULL. */
const char* gpa_last_error(void);

/* Library version string, e.g. "gpapriori-b200 0.1 sm_100a". */
const char* gpa_version(void);

/* Number of GPU kernels this library has launched in the process so far (all devices, all
 * threads; includes the CUB scan kernels of the device level transition).  Instrumentation for
 * benchmarks: the difference across a timed region is the kernel-launch count of that region. */
uint64_t gpa_kernel_launches(void);

/* ------------------------------------------------------------------ inputs */

#define GPA_MEM_HOST 0u        /* offsets/items are host pointers (pinned or pageable) */
#define GPA_MEM_DEVICE 1u      /* offsets/items are device pointers on the library's device */

/*
 * Horizontal transaction database in CSR form ("store a list of items that comprise each
 * transaction ... the horizontal representation", P13@1530).
 *   n_tx      number of transactions N (empty transactions are allowed and count in N);
 *   offsets   n_tx+1 entries, offsets[0] == 0, non-decreasing; transaction t is
 *             items[offsets[t] .. offsets[t+1]);
 *   items     offsets[n_tx] item ids, each < n_items; order inside a transaction is free and
 *             duplicates are ignored (a transaction is a set, P3@441; Q4);
 *   n_items   size of the item-id universe;
 *   memory    GPA_MEM_HOST or GPA_MEM_DEVICE.
 * With a gpa_dist, each rank passes its own contiguous transaction range; ranges are in rank
 * order and every range except the last holds a multiple of 512 transactions.
 */
typedef struct {
  uint64_t n_tx;
  const uint64_t* offsets;
  const uint32_t* items;
  uint32_t n_items;
  uint32_t memory;
} gpa_tx_csr;

/* Counting kernel selection. */
#define GPA_KERNEL_AUTO 0u     /* gpa_mine: PAIRS_TC for k = 2, PROJ for k >= 3 (TRIE / PREFIX if the projected
                                  lists do not fit); gpa_count: TRIE for 3 <= k <= 16, PREFIX above */
#define GPA_KERNEL_V0 1u       /* the paper's design: one CTA per candidate, AND of all k rows */
#define GPA_KERNEL_PREFIX 2u   /* prefix-staged streaming: (k-1)-prefix AND held on chip, siblings streamed */
#define GPA_KERNEL_PAIRS 3u    /* k = 2 only: TMA-tiled AND-popcount "Gram" tile kernel */
#define GPA_KERNEL_TRIE 4u     /* 2 <= k <= 16: transaction-tiled trie walk, rows staged in shared memory */
#define GPA_KERNEL_PAIRS_TC 5u /* k = 2 only: the pair Gram B B^T of the 0/1 rows as a tcgen05 integer GEMM
                                  (kind::i8, s32 accumulators in TMEM); exact, same counts as PAIRS */
#define GPA_KERNEL_PROJ 6u     /* gpa_mine, k >= 3: "equivalent class clustering" (P13@2288-2486) on projected
                                  vertical lists -- each L_{k-1} member keeps its last item's bits restricted
                                  to the transactions of its (k-2)-prefix; a candidate's support is the
                                  popcount of the AND of its two parents' lists (exact, same counts as
                                  complete intersection).  k = 2 as AUTO; gpa_count treats it as AUTO */
#define GPA_KERNEL_FUSED 7u    /* gpa_mine: every generation k >= 2 in ONE cooperative launch (grid-wide phases:
                                  complete-intersection counting, threshold, join + prune; no per-level launch or
                                  host round trip) when |L_1| <= 1,024 and the L_1 rows fit 48 MB; AUTO picks it for
                                  such problems on one GPU.  Otherwise (or on a capacity overflow) AUTO's kernels.
                                  gpa_count treats it as AUTO */

#define GPA_KEEP_CANDIDATES 1u /* gpa_mine: keep every generation's (C_k, counts), not only F */
#define GPA_HOST_CANDGEN 2u    /* gpa_mine: join + prune on the host thread pool instead of the device
                                  (reference path; the default keeps the level transition on the GPU) */
#define GPA_NO_OVERLAP_INGEST 4u /* gpa_mine, host input: upload the whole database before computing
                                  (default: upload in chunks overlapped with histogram, bitset build and
                                  generation-2 counting) */
#define GPA_MULTI_KERNEL 16u    /* gpa_mine: never the single-launch path of GPA_KERNEL_FUSED under AUTO */
#define GPA_COMPLETE_INTERSECTION 8u /* gpa_mine: every generation k >= 3 by complete intersection from the
                                  static bitset (the paper's method, P18@394; TRIE / PREFIX kernels), never
                                  the projected lists of GPA_KERNEL_PROJ.  With count_kernel GPA_KERNEL_PAIRS
                                  this is the north-star path without tensor cores */

typedef struct {
  uint32_t count_kernel;       /* GPA_KERNEL_*; default GPA_KERNEL_AUTO */
  uint32_t flags;              /* GPA_KEEP_CANDIDATES | ... ; default 0 */
  void* stream;                /* cudaStream_t to run on; NULL = a library-owned stream */
  int32_t device;              /* CUDA device ordinal; -1 = the calling thread's current device */
  uint32_t max_k;              /* gpa_mine: stop after this generation (0 = no limit, <= GPA_MAX_K) */
  uint32_t reserved[3];        /* must be zero */
} gpa_options;

/* Fill *opt with the defaults above. */
void gpa_options_default(gpa_options* opt);

/* Exact threshold: max(1, ceil(n_tx * num / den)) for a support ratio num/den (P4@0, P4@111;
 * DESIGN.md Q2).  Returns 0 if den == 0. */
uint64_t gpa_min_count(uint64_t n_tx, uint64_t num, uint64_t den);

/* ------------------------------------------------------------------ multi-GPU */

/*
 * One process per GPU; the transaction dimension is sharded across ranks and every count
 * vector is summed with an NCCL all-reduce over NVLink.
 * gpa_dist_unique_id runs on one rank (wraps ncclGetUniqueId); the 128 bytes are broadcast
 * by the caller (e.g. torch.distributed) and every rank calls gpa_dist_create collectively.
 */
typedef struct gpa_dist gpa_dist;
gpa_status gpa_dist_unique_id(uint8_t id_out[128]);
gpa_status gpa_dist_create(int rank, int world, int device, const uint8_t id[128], gpa_dist** out);
gpa_status gpa_dist_destroy(gpa_dist* dist);
/* rank / world of a communicator (for bindings and tests). */
gpa_status gpa_dist_info(const gpa_dist* dist, int* rank, int* world);

/*
 * Host-staged collectives: the same sharded path (every all-reduce of gpa_bitset_create /
 * gpa_count / gpa_mine, in the same order and sizes) over a caller-supplied in-place
 * all-reduce of HOST memory -- for ranks that share one GPU (NCCL refuses two ranks on one
 * device), for MPI / gloo users, and for tests of the sharded path.  Each collective copies
 * the device buffer to a pinned host buffer, synchronises the stream, calls
 *     fn(ctx, host_buf, n, dtype, op)   dtype: GPA_DT_U32 / GPA_DT_U64, op: GPA_OP_SUM / GPA_OP_MAX
 * which must leave the element-wise reduction over all ranks in host_buf and return 0 (any
 * other value fails the call with GPA_ERR_NCCL and marks the handle unusable, GPA_ERR_STATE),
 * then copies the result back.  fn is called on the thread that called the library.
 */
#define GPA_DT_U32 0u
#define GPA_DT_U64 1u
#define GPA_OP_SUM 0u
#define GPA_OP_MAX 1u
typedef int (*gpa_host_allreduce_fn)(void* ctx, void* host_buf, uint64_t n, uint32_t dtype, uint32_t op);
gpa_status gpa_dist_create_host(int rank, int world, int device, gpa_host_allreduce_fn fn, void* ctx,
                                gpa_dist** out);

/*
 * Collective log: every all-reduce this handle has issued, in order, encoded as
 * (op << 60) | (dtype << 56) | n.  *n_total = the number issued; min(cap, *n_total) entries are
 * written to entries (may be NULL when cap == 0).  Every rank of a correct run issues the same
 * sequence -- the library takes every path decision (overlapped ingest, fallbacks, input
 * validation) collectively, so the sequences never diverge (tests compare them).
 */
gpa_status gpa_dist_log(const gpa_dist* dist, uint64_t* entries, uint64_t cap, uint64_t* n_total);

/*
 * Failure detection (NCCL): waits on the library's streams poll ncclCommGetAsyncError; an
 * asynchronous NCCL error, or a wait longer than `seconds` (default 600; <= 0 disables), aborts the
 * communicator (ncclCommAbort) and fails the call with GPA_ERR_NCCL; the handle then reports
 * GPA_ERR_STATE.
 */
gpa_status gpa_dist_set_timeout(gpa_dist* dist, double seconds);

/* ------------------------------------------------------------------ static bitset */

/*
 * Build the static bitset of db on the device: one row per item whose (global) count is
 * >= row_min_count (row_min_count = 1: every occurring item; = min_count: the paper's
 * "vertical lists of first generation", P18@755; = 0: every item id < n_items, absent items
 * with an all-zero row).  Rows are ordered by ascending item id.
 * Row r, transaction t -> word t/32, bit t%32 (LSB first; Q9); padding bits are 0;
 * the row pitch is a multiple of 128 bytes (>= the paper's 64-byte alignment, P18@1685).
 * With dist, the call is collective; each rank holds the rows over its own transactions and
 * the item counts are global.  opt may be NULL (defaults).
 */
typedef struct gpa_bitset gpa_bitset;
gpa_status gpa_bitset_create(const gpa_tx_csr* db, uint32_t row_min_count, const gpa_dist* dist,
                             const gpa_options* opt, gpa_bitset** out);
gpa_status gpa_bitset_destroy(gpa_bitset* bs);

/* n_tx_local: this rank's transactions; n_tx_global: all ranks; n_rows; row_pitch_bytes. */
gpa_status gpa_bitset_info(const gpa_bitset* bs, uint64_t* n_tx_local, uint64_t* n_tx_global,
                           uint32_t* n_rows, uint64_t* row_pitch_bytes);

/* Global item counts (the generation-1 supports, P13@338): counts_out[n_items], host. */
gpa_status gpa_bitset_item_counts(const gpa_bitset* bs, uint32_t* counts_out);

/* Item id owning each row: item_of_row_out[n_rows], host, ascending. */
gpa_status gpa_bitset_rows(const gpa_bitset* bs, uint32_t* item_of_row_out);

/* Copy this rank's rows to host: host_out[n_rows * row_pitch_bytes/4] words. */
gpa_status gpa_bitset_export(const gpa_bitset* bs, uint32_t* host_out);

/*
 * Supports of M candidates of k items each (cand: host, M*k ORIGINAL item ids, each row
 * strictly increasing; any row order): counts_out[m] = popcount(AND of the k rows of
 * candidate m) = supp(candidate m), summed over ranks with dist (collective).
 * 1 <= k <= GPA_MAX_K.  M == 0 is a no-op.  kernel: GPA_KERNEL_* (AUTO honours the options
 * the bitset was created with).  GPA_ERR_RANGE if an item has no row.
 */
gpa_status gpa_count(gpa_bitset* bs, const uint32_t* cand, uint32_t k, uint64_t M, uint32_t kernel,
                     uint32_t* counts_out);

/* ------------------------------------------------------------------ level-wise mining */

/*
 * Level-wise Apriori (P13@338-652) with GPU support counting: generation 1 by a device
 * histogram, the static bitset of the frequent items, then for k = 2, 3, ...:
 * C_k = join + prune of L_{k-1} (trie leaf-sibling join P13@1006-1270, prune by downward
 * closure P13@178), grouped by (k-1)-prefix; supports by complete intersection on the GPU;
 * L_k = { c : count >= min_count }.  Stops when L_k or C_{k+1} is empty (P13@652) or after
 * opt->max_k.  Result: F = all (itemset, support) with support >= min_count in original item
 * ids; with GPA_KEEP_CANDIDATES also every (C_k, counts).  Collective with dist.
 */
typedef struct gpa_result gpa_result;
gpa_status gpa_mine(const gpa_tx_csr* db, uint64_t min_count, const gpa_dist* dist, const gpa_options* opt,
                    gpa_result** out);

/* N (global transaction count, all ranks) and the min_count the result was mined with. */
gpa_status gpa_result_info(const gpa_result* r, uint64_t* n_tx, uint64_t* min_count);

/* Number of frequent itemsets |F| and the longest frequent itemset length. */
gpa_status gpa_result_count(const gpa_result* r, uint64_t* n_itemsets, uint32_t* max_k);

/* i-th frequent itemset in canonical order (by k, then lexicographic by item id). */
gpa_status gpa_result_get(const gpa_result* r, uint64_t i, const uint32_t** items, uint32_t* k, uint32_t* support);

/* All frequent k-itemsets at once: *items -> n*k ids (lexicographic rows), *supports -> n. */
gpa_status gpa_result_frequent(const gpa_result* r, uint32_t k, uint64_t* n, const uint32_t** items,
                               const uint32_t** supports);

/* Generation k (k >= 1): |C_k| and |L_k|; with GPA_KEEP_CANDIDATES also the candidates
 * (n_cand*k ids, lexicographic) and their counts, else *cand = *counts = NULL.
 * GPA_ERR_RANGE if generation k was not reached. */
gpa_status gpa_result_level(const gpa_result* r, uint32_t k, uint64_t* n_cand, uint64_t* n_freq,
                            const uint32_t** cand, const uint32_t** counts);

/* Number of generations run (1 + the number of counted candidate generations). */
gpa_status gpa_result_n_levels(const gpa_result* r, uint32_t* n_levels);

/* Per-generation statistics of the counting step. */
typedef struct {
  uint64_t n_cand;             /* |C_k| */
  uint64_t n_freq;             /* |L_k| */
  uint64_t n_groups;           /* (k-1)-prefix groups */
  uint32_t kernel;             /* GPA_KERNEL_* that ran */
  uint32_t launches;           /* counting kernel launches */
  double count_ms;             /* CUDA-event time of the counting kernel(s), this rank */
  double allreduce_ms;         /* CUDA-event time of the count all-reduce (0 without dist) */
  double candgen_ms;           /* host join + prune + grouping */
  double build_ms;             /* GPA_KERNEL_PROJ: CUDA-event time of the list-building kernel (pext) for
                                  L_{k-1}'s projected lists (included in count_ms); 0 otherwise */
  uint64_t build_words;        /* GPA_KERNEL_PROJ: 32-bit mask words x members the list build compressed
                                  (its algorithmic work); 0 otherwise */
  double setup_ms;             /* GPA_KERNEL_PROJ: CUDA-event time from the start of the generation's
                                  counting to the list-building kernel (class tables, sizes); the
                                  support kernel is count_ms - setup_ms - build_ms */
  uint64_t build_bytes;        /* GPA_KERNEL_PROJ: algorithmic HBM bytes of the list build: every source
                                  list (generation 3: bitset row) read once + the new lists written once */
  uint64_t count_bytes;        /* GPA_KERNEL_PROJ: algorithmic HBM bytes of the support kernel: every list
                                  of L_{k-1} read once + the counts written */
} gpa_level_stats;
gpa_status gpa_result_level_stats(const gpa_result* r, uint32_t k, gpa_level_stats* out);

/* Phase times in milliseconds.  UPLOAD .. BITSET: host wall clock around each (synchronised)
 * build phase; CANDGEN, COUNT, THRESHOLD: CUDA-event time on the mining stream, generation by
 * generation (contiguous: their sum is the level loop's device timeline); TOTAL: wall clock. */
#define GPA_PHASE_UPLOAD 0     /* H2D of the CSR (host input only; overlapped ingest: upload + histogram +
                                  bitset + generation-2 counting of the chunks) */
#define GPA_PHASE_HISTOGRAM 1  /* validation + generation-1 counts (+ all-reduce) */
#define GPA_PHASE_BITSET 2     /* static bitset build */
#define GPA_PHASE_CANDGEN 3    /* join + prune of C_k (+ class tables of the projected lists) */
#define GPA_PHASE_COUNT 4      /* list build + counting kernels + all-reduce */
#define GPA_PHASE_THRESHOLD 5  /* L_k selection + compaction + item mapping */
#define GPA_PHASE_TOTAL 6      /* whole gpa_mine call */
#define GPA_PHASE_COUNT_ 7
gpa_status gpa_result_timing(const gpa_result* r, double ms_by_phase[GPA_PHASE_COUNT_]);

gpa_status gpa_result_destroy(gpa_result* r);

/* ------------------------------------------------------------------ association rules (f4) */

/*
 * Association rules from a mining result -- the downstream use of frequent itemsets that the paper
 * motivates (P4@338-720, "people who buy vegetables often also buy salad dressing"); the paper
 * does not define them, the reading (Q19) is Agrawal & Srikant's (ref [2], P28@1007):
 * for every frequent X with |X| >= 2 and every non-empty proper subset A of X, the rule
 * A => X \ A is reported iff  supp(X) / supp(A) >= conf_num / conf_den, decided exactly as
 * supp(X) * conf_den >= conf_num * supp(A) (64-bit integers).  Computed on the current CUDA device.
 *
 * Rule j: X = itemset number itemset[j] of the result (the index of gpa_result_get, canonical
 * order), antecedent A = the items of X whose bit is set in antecedent_mask[j] (bit q = X's q-th
 * item), consequent = the others; support of the rule = supp(X), antecedent_support[j] = supp(A).
 * Rules come ordered by itemset index, then by mask.  Errors: GPA_ERR_INVALID (NULL, conf_den == 0),
 * GPA_ERR_RANGE (an itemset longer than GPA_RULES_MAX_K, or more than 2^32 rules).  The arrays are
 * owned by the gpa_rules handle (valid until gpa_rules_destroy; the result may be destroyed first).
 */
#define GPA_RULES_MAX_K 20u
typedef struct gpa_rules gpa_rules;
gpa_status gpa_rules_create(const gpa_result* r, uint64_t conf_num, uint64_t conf_den, gpa_rules** out);
gpa_status gpa_rules_arrays(const gpa_rules* rules, uint64_t* n_rules, const uint32_t** itemset,
                            const uint32_t** antecedent_mask, const uint32_t** antecedent_support);
gpa_status gpa_rules_destroy(gpa_rules* rules);

#ifdef __cplusplus
}
#endif

#endif /* GPAPRIORI_H */
