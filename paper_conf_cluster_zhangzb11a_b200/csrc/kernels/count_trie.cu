// count_trie -- support counting for generations k >= 3 as a transaction-tiled trie walk (sm_100a).
//
// Complete intersection (PAPER.md P18@394-1300): supp(c) = sum_w popc(B[c_1][w] & ... & B[c_k][w]).
// The candidates of a generation, in lexicographic order, are the leaves of the candidate trie
// (P13@835-1270, Fig. 1 / Fig. 4); consecutive candidates share prefixes, so the AND of a shared
// prefix is computed once and reused ("candidates from the k-th and (k+1)-th generation share the
// same prefix").  Deep generations have tiny sibling groups (mean 2-5), so the win comes from
// reusing loaded words across MANY candidates, not only siblings:
//
//   * the host cuts the candidate list into BLOCKS of <= 256 lexicographically consecutive
//     candidates touching <= 32 distinct rows (64 for k = 2); each of the 8 warps of a CTA owns
//     32 of them;
//   * a CTA = (block, part of the transaction axis).  It streams its part in STRIPES of 128 x W
//     words (W = 2 for k >= 3, 1 for k = 2): a producer warp brings the block's rows' segments into a
//     shared-memory ring with 1-D bulk async copies (cp.async.bulk + mbarrier complete_tx);
//   * the 8 consumer warps split the block's candidates evenly and walk them for every stripe:
//     lane = 8 words (2 independent LDS.128 per row, conflict-free); the deepest three levels of
//     the prefix stack V[d] = AND of the first d+1 rows live in registers and are recomputed only
//     from the first position where a candidate differs from its predecessor (lcp; a warp-uniform
//     jump into an unrolled fall-through chain, so skipped levels cost nothing); shallower levels
//     are folded from shared memory when a candidate changes them (rare), which keeps the kernel
//     at 72 registers = 3 CTAs (27 warps) per SM for every k;
//   * the leaf is 2 LDS.128 + 8 AND + 8 POPC per lane, reduced across the warp with redux.sync;
//     lane j keeps candidate j's running count in a register (the reduced value is added one
//     candidate later, and the next candidate's descriptor is loaded one candidate ahead, so
//     neither latency sits on the critical path).  Compact, non-unrolled candidate loop: no
//     I-cache thrash.  The bitset pitch is a multiple of the 256-word stripe: no ragged stripe;
//   * only after the whole part: one atomicAdd per (CTA, candidate).
// Work per cand x word: ~1 LDS word + 1 AND + 1 POPC + (lcp recompute); no per-stripe reductions
// to memory, no global traffic besides the row segments (DRAM ~ the bitset once per part-window;
// the grid is part-major so concurrently running CTAs share the same stripes in L2).  Measured
// bound (ncu, k = 6, 7): shared-memory bandwidth (~80%) with POPC issue at 62-68%.
// Tried and rejected (slower): 16 words per lane at 2 CTAs/SM (k >= 7 +40%);
// a per-class program keeping V_Q & R_a for 4 anchors in registers (half the row loads, but
// +25% instructions and warp imbalance: +50%).
#include <cstdint>
#include "../common.h"
#include "../kernels.h"

namespace gpa {
namespace {

constexpr int kWarps = 8;                          // consumer warps
constexpr int kThreads = (kWarps + 1) * 32;        // + 1 producer warp (bulk copies)
constexpr int kCandPerWarp = 32;
constexpr uint32_t kTrieMaxStages = 8;
constexpr uint32_t kTrieRingBytes = 64u * 1024u;   // stripe ring per CTA (3 CTAs / SM)

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

__device__ __forceinline__ void mbar_init(uint32_t bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(bar), "r"(count));
}
__device__ __forceinline__ void mbar_arrive_expect_tx(uint32_t bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint32_t bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(bar) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint32_t bar, uint32_t parity) {
  asm volatile(
      "{\n"
      ".reg .pred P1;\n"
      "LAB_WAIT:\n"
      "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n"
      "@P1 bra DONE;\n"
      "bra LAB_WAIT;\n"
      "DONE:\n"
      "}\n" ::"r"(bar),
      "r"(parity)
      : "memory");
}
__device__ __forceinline__ void bulk_g2s(uint32_t dst, const void* src, uint32_t bytes, uint32_t bar) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(dst),
               "l"(src), "r"(bytes), "r"(bar)
               : "memory");
}
__device__ __forceinline__ uint4 lds128(uint32_t addr) {
  uint4 v;
  asm volatile("ld.shared.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "r"(addr));
  return v;
}
__device__ __forceinline__ uint4 and4(const uint4& a, const uint4& b) {
  return make_uint4(a.x & b.x, a.y & b.y, a.z & b.z, a.w & b.w);
}

// byte offset (local row * segment bytes) of level d in the candidate's descriptor: 16-bit
// fields, levels 0-7 in lo, 8-15 in hi.  Segments are >= 512 B, so the low 5 bits of level 0's
// field are free: they carry the candidate's lcp (kLcpMask).
constexpr uint32_t kLcpMask = 31u;
__device__ __forceinline__ uint32_t off_of(const uint4& lo, const uint4& hi, int d) {
  const uint4& v = d < 8 ? lo : hi;
  const int e = d & 7;
  const uint32_t w = e < 2 ? v.x : e < 4 ? v.y : e < 6 ? v.z : v.w;
  return (e & 1) ? (w >> 16) : (w & (d == 0 ? 0xffffu & ~kLcpMask : 0xffffu));
}

// Register-resident prefix levels: only the deepest kTrieRegLevels levels of the stack V live in
// registers (V[i] = AND of rows 0..D0+i, D0 = K-1-kTrieRegLevels); a candidate whose shared prefix
// with its predecessor is shorter than D0 (a new (K-3)-prefix: ~10-20% of candidates at deep
// generations) folds rows 0..D0 from shared memory again.  This keeps the stack at 3 x W uint4 for
// every K: 72 registers, 3 CTAs (27 warps) per SM, W = 2 up to K = 16.
template <int K>
constexpr int kTrieRegLevels = K - 1 < 3 ? K - 1 : 3;

// Level D (>= D0) of the stack: V[D-D0] = V[D-D0-1] & row_D, or the fold of rows 0..D0 for D = D0.
template <int K, int W, int D>
__device__ __forceinline__ void trie_level(uint4 (&V)[kTrieRegLevels<K>][W], uint32_t base, const uint4& lo,
                                           const uint4& hi) {
  constexpr int D0 = K - 1 - kTrieRegLevels<K>;
  if constexpr (D >= D0 && D < K - 1) {
    if constexpr (D == D0) {
      uint4 v[W];
      const uint32_t a0 = base + off_of(lo, hi, 0);
#pragma unroll
      for (int u = 0; u < W; ++u) v[u] = lds128(a0 + u * 512);
#pragma unroll
      for (int d = 1; d <= D0; ++d) {
        const uint32_t a = base + off_of(lo, hi, d);
#pragma unroll
        for (int u = 0; u < W; ++u) v[u] = and4(v[u], lds128(a + u * 512));
      }
#pragma unroll
      for (int u = 0; u < W; ++u) V[0][u] = v[u];
    } else {
      const uint32_t a = base + off_of(lo, hi, D);
      uint4 v[W];
#pragma unroll
      for (int u = 0; u < W; ++u) v[u] = lds128(a + u * 512);
#pragma unroll
      for (int u = 0; u < W; ++u) V[D - D0][u] = and4(V[D - D0 - 1 >= 0 ? D - D0 - 1 : 0][u], v[u]);
    }
  }
}

template <int K, int W>
__global__ void __launch_bounds__(kThreads, 3) count_trie_kernel(
    const uint32_t* __restrict__ rows, uint64_t pitch_words, const TrieBlock* __restrict__ blocks,
    const uint32_t* __restrict__ block_rows, const uint4* __restrict__ cand_lrows, const uint8_t* __restrict__ cand_lcp,
    uint32_t n_blocks, uint32_t n_parts, uint32_t n_stripes, uint32_t n_stages, uint32_t* __restrict__ counts) {
  constexpr uint32_t kStripeWords = 128 * W;
  constexpr uint32_t kSegBytes = kStripeWords * 4;
  constexpr int R = kTrieRegLevels<K>;
  constexpr int D0 = K - 1 - R;
  extern __shared__ __align__(16) uint8_t smem[];
  __shared__ uint4 s_desc[kWarps * kCandPerWarp][K > 8 ? 2 : 1];
  __shared__ uint32_t s_rowid[kTrieMaxRows];
  __shared__ __align__(8) uint64_t s_full[kTrieMaxStages];
  __shared__ __align__(8) uint64_t s_empty[kTrieMaxStages];

  const uint32_t b = blockIdx.x % n_blocks;
  const uint32_t part = blockIdx.x / n_blocks;
  const TrieBlock blk = blocks[b];
  const uint32_t st0 = (uint32_t)((uint64_t)n_stripes * part / n_parts);
  const uint32_t st1 = (uint32_t)((uint64_t)n_stripes * (part + 1) / n_parts);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;

  // descriptor: 16-bit shared-memory offsets of the candidate's rows (local row * segment bytes)
  for (uint32_t i = threadIdx.x; i < blk.n_cand; i += kThreads) {
    const uint4 lr = cand_lrows[blk.cand_begin + i];
    const uint32_t w[4] = {lr.x, lr.y, lr.z, lr.w};
    uint32_t o[8];
#pragma unroll
    for (int q = 0; q < 8; ++q) {
      const uint32_t b0 = (w[q >> 1] >> (16 * (q & 1))) & 0xffu, b1 = (w[q >> 1] >> (16 * (q & 1) + 8)) & 0xffu;
      o[q] = (b0 * kSegBytes) | ((b1 * kSegBytes) << 16);
    }
    s_desc[i][0] = make_uint4(o[0] | cand_lcp[blk.cand_begin + i], o[1], o[2], o[3]);
    if constexpr (K > 8) s_desc[i][K > 8 ? 1 : 0] = make_uint4(o[4], o[5], o[6], o[7]);
  }
  for (uint32_t i = threadIdx.x; i < blk.n_rows; i += kThreads) s_rowid[i] = block_rows[blk.row_begin + i];
  const uint32_t full0 = smem_u32(&s_full[0]);
  const uint32_t empty0 = smem_u32(&s_empty[0]);
  if (threadIdx.x == 0) {
    for (uint32_t q = 0; q < n_stages; ++q) {
      mbar_init(full0 + 8 * q, 1);
      mbar_init(empty0 + 8 * q, kWarps);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  if (st0 >= st1) return;

  const uint32_t buf0 = smem_u32(smem);
  const uint32_t buf_bytes = blk.n_rows * kSegBytes;

  if (warp == kWarps) {
    // ---------------- producer warp: stripe s -> ring slot i % n_stages, one bulk copy per row
    for (uint32_t s = st0, i = 0; s < st1; ++s, ++i) {
      const uint32_t slot = i % n_stages;
      mbar_wait(empty0 + 8 * slot, ((i / n_stages) & 1) ^ 1);
      const uint32_t bar = full0 + 8 * slot;
      const uint64_t w0 = (uint64_t)s * kStripeWords;
      if (lane == 0) mbar_arrive_expect_tx(bar, kSegBytes * blk.n_rows);
      __syncwarp();
      const uint32_t dst = buf0 + slot * buf_bytes;
      for (uint32_t r = lane; r < blk.n_rows; r += 32)
        bulk_g2s(dst + r * kSegBytes, rows + (uint64_t)s_rowid[r] * pitch_words + w0, kSegBytes, bar);
    }
    return;
  }

  // ---------------- consumer warps: the block's candidates split evenly, <= 32 per warp.
  // Lane j accumulates candidate my0 + j over all stripes of the part (register, no shared-memory
  // counters).
  const int chunk = ((int)blk.n_cand + kWarps - 1) / kWarps;
  const int my0 = warp * chunk;
  const int n_mine = max(0, min(chunk, (int)blk.n_cand - my0));
  uint32_t acc = 0;
  uint4 V[R][W];
#pragma unroll
  for (int d = 0; d < R; ++d)
#pragma unroll
    for (int u = 0; u < W; ++u) V[d][u] = make_uint4(0, 0, 0, 0);

  // one candidate: recompute the stack from the first level that differs from the previous
  // candidate (warp-uniform; a sibling (lcp = K-1) only needs the leaf, a cousin (K-2) one
  // level), then this lane's popcount of the leaf AND
  auto candidate = [&](uint32_t base, const uint4& lo, const uint4& hi) -> uint32_t {
    const int l = lo.x & kLcpMask;
    if (l <= K - 2) {
      if (l <= K - 3) {
        switch (l < D0 ? D0 : l) {
#define GPA_TRIE_LEVEL(D) \
  case D:                 \
    if constexpr (D <= K - 3) trie_level<K, W, D>(V, base, lo, hi); [[fallthrough]];
          GPA_TRIE_LEVEL(0) GPA_TRIE_LEVEL(1) GPA_TRIE_LEVEL(2) GPA_TRIE_LEVEL(3) GPA_TRIE_LEVEL(4)
          GPA_TRIE_LEVEL(5) GPA_TRIE_LEVEL(6) GPA_TRIE_LEVEL(7) GPA_TRIE_LEVEL(8) GPA_TRIE_LEVEL(9)
          GPA_TRIE_LEVEL(10) GPA_TRIE_LEVEL(11) GPA_TRIE_LEVEL(12) GPA_TRIE_LEVEL(13)
#undef GPA_TRIE_LEVEL
          default:
            break;
        }
      }
      trie_level<K, W, K - 2>(V, base, lo, hi);
    }
    const uint32_t a = base + off_of(lo, hi, K - 1);
    uint4 v[W];
#pragma unroll
    for (int u = 0; u < W; ++u) v[u] = lds128(a + u * 512);
    uint32_t c = 0;
#pragma unroll
    for (int u = 0; u < W; ++u)
      c += (__popc(V[R - 1][u].x & v[u].x) + __popc(V[R - 1][u].y & v[u].y)) +
           (__popc(V[R - 1][u].z & v[u].z) + __popc(V[R - 1][u].w & v[u].w));
    return c;
  };

  for (uint32_t s = st0, i = 0; s < st1; ++s, ++i) {
    const uint32_t slot = i % n_stages;
    mbar_wait(full0 + 8 * slot, (i / n_stages) & 1);
    const uint32_t base = buf0 + slot * buf_bytes + lane * 16;
    // candidates in pairs: both lane partials (<= 32 x 8 x 32 = 8,192 summed over the warp) share
    // one redux.sync, packed into 16-bit halves
#pragma unroll 1
    for (int j = 0; j < n_mine; j += 2) {
      const bool two = j + 1 < n_mine;
      const uint4 lo0 = s_desc[my0 + j][0];
      const uint4 hi0 = K > 8 ? s_desc[my0 + j][K > 8 ? 1 : 0] : make_uint4(0, 0, 0, 0);
      const uint4 lo1 = s_desc[my0 + j + (two ? 1 : 0)][0];
      const uint4 hi1 = K > 8 ? s_desc[my0 + j + (two ? 1 : 0)][K > 8 ? 1 : 0] : make_uint4(0, 0, 0, 0);
      uint32_t c = candidate(base, lo0, hi0);
      if (two) c |= candidate(base, lo1, hi1) << 16;
      c = __reduce_add_sync(0xffffffffu, c);
      acc += lane == j ? (c & 0xffffu) : (lane == j + 1 ? (c >> 16) : 0u);
    }
    __syncwarp();
    if (lane == 0) mbar_arrive(empty0 + 8 * slot);
  }
  if (lane < n_mine && acc) atomicAdd(&counts[blk.cand_begin + my0 + lane], acc);
}

template <int K, int W>
void launch_k(const uint32_t* rows, uint64_t pitch_words, const TrieBlock* blocks, const uint32_t* block_rows,
              const uint4* lrows, const uint8_t* lcp, uint32_t n_blocks, uint32_t n_parts, uint32_t max_rows,
              uint32_t* counts, cudaStream_t stream) {
  constexpr uint32_t kSegBytes = 512 * W;
  const uint32_t n_stripes = (uint32_t)(pitch_words / (128 * W));
  if (n_parts > n_stripes) n_parts = n_stripes;
  if (n_parts < 1) n_parts = 1;
  // ring depth: as many stripes in flight as fit the ring budget (3 or 2 CTAs / SM), 2..kTrieMaxStages
  uint32_t stages = (uint32_t)(kTrieRingBytes / ((size_t)max_rows * kSegBytes));
  stages = stages < 2 ? 2 : (stages > kTrieMaxStages ? kTrieMaxStages : stages);
  const size_t smem = (size_t)stages * max_rows * kSegBytes;
  ensure_smem_attr(reinterpret_cast<const void*>(count_trie_kernel<K, W>), 200 * 1024);
  const uint64_t grid = (uint64_t)n_blocks * n_parts;
  GPA_REQUIRE(grid < (1ull << 31), GPA_ERR_INVALID, "count_trie: grid too large");
  { count_trie_kernel<K, W><<<(unsigned)grid, kThreads, smem, stream>>>(rows, pitch_words, blocks, block_rows, lrows,
                                                                      lcp, n_blocks, n_parts, n_stripes, stages, counts); note_launch(); }
  GPA_CUDA(cudaGetLastError());
}

}  // namespace

uint64_t launch_count_trie(uint32_t k, const uint32_t* rows, uint64_t pitch_words, const TrieBlock* blocks,
                           const uint32_t* block_rows, const uint4* cand_lrows, const uint8_t* cand_lcp,
                           uint32_t n_blocks, uint32_t max_rows, uint32_t n_parts, uint32_t* counts,
                           cudaStream_t stream) {
  if (n_blocks == 0) return 0;
  GPA_REQUIRE(max_rows <= trie_max_rows(k), GPA_ERR_INVALID, "count_trie: block with %u rows", max_rows);
#define GPA_TRIE_CASE(KK, WW)                                                                                     \
  case KK:                                                                                                       \
    launch_k<KK, WW>(rows, pitch_words, blocks, block_rows, cand_lrows, cand_lcp, n_blocks, n_parts, max_rows,   \
                     counts, stream);                                                                            \
    break;
  switch (k) {
    GPA_TRIE_CASE(2, 1) GPA_TRIE_CASE(3, 2) GPA_TRIE_CASE(4, 2) GPA_TRIE_CASE(5, 2) GPA_TRIE_CASE(6, 2)
    GPA_TRIE_CASE(7, 2) GPA_TRIE_CASE(8, 2) GPA_TRIE_CASE(9, 2) GPA_TRIE_CASE(10, 2) GPA_TRIE_CASE(11, 2)
    GPA_TRIE_CASE(12, 2) GPA_TRIE_CASE(13, 2) GPA_TRIE_CASE(14, 2) GPA_TRIE_CASE(15, 2) GPA_TRIE_CASE(16, 2)
    default:
      fail(GPA_ERR_INVALID, "count_trie: k = %u outside [2, %u]", k, kTrieMaxK);
  }
#undef GPA_TRIE_CASE
  return (uint64_t)n_blocks * n_parts;
}

}  // namespace gpa
