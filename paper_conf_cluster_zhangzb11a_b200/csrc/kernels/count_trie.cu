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
//     candidates touching <= 64 distinct rows; each of the 8 warps of a CTA owns 32 of them;
//   * a CTA = (block, part of the transaction axis).  It streams its part in STRIPES of 128
//     words (4,096 transactions): the block's rows' 512-byte segments are brought into shared
//     memory by 1-D bulk async copies (cp.async.bulk + mbarrier complete_tx), double buffered;
//   * every warp walks its 32 candidates for the stripe: lane = 4 consecutive words (LDS.128,
//     conflict-free); a register stack V[d] = AND of the first d+1 rows is recomputed only from
//     the first position where a candidate differs from its predecessor (lcp), the leaf is one
//     LDS.128 + 4 AND + 4 POPC into a per-candidate REGISTER accumulator;
//   * only after the whole part: warp reduction (redux.sync) + one atomicAdd per (CTA, candidate).
// Work per cand x word: ~1 LDS word + 1 AND + 1 POPC + (lcp recompute); no per-stripe reductions,
// no global traffic besides the row segments (DRAM ~ the bitset once per part-window, the grid is
// part-major so concurrently running CTAs share the same stripes in L2).  Bound: POPC issue.
#include <cstdint>
#include "../common.h"
#include "../kernels.h"

namespace gpa {
namespace {

constexpr int kThreads = 256;
constexpr int kWarps = kThreads / 32;
constexpr int kCandPerWarp = 32;
constexpr int kStripeWords = 128;                 // 32 lanes x 4 words
constexpr int kSegBytes = kStripeWords * 4;       // 512 B per row segment

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

__device__ __forceinline__ void mbar_init(uint32_t bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(bar), "r"(count));
}
__device__ __forceinline__ void mbar_arrive_expect_tx(uint32_t bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes) : "memory");
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
__device__ __forceinline__ uint32_t byte_of(const uint4& v, int d) {
  const uint32_t w = d < 4 ? v.x : d < 8 ? v.y : d < 12 ? v.z : v.w;
  return (w >> (8 * (d & 3))) & 0xffu;
}

template <int K>
__global__ void __launch_bounds__(kThreads, 2) count_trie_kernel(
    const uint32_t* __restrict__ rows, uint64_t pitch_words, const TrieBlock* __restrict__ blocks,
    const uint32_t* __restrict__ block_rows, const uint4* __restrict__ cand_lrows, const uint8_t* __restrict__ cand_lcp,
    uint32_t n_blocks, uint32_t n_parts, uint32_t n_stripes, uint32_t* __restrict__ counts) {
  extern __shared__ __align__(16) uint8_t smem[];
  __shared__ uint4 s_lrows[kWarps * kCandPerWarp];
  __shared__ uint8_t s_lcp[kWarps * kCandPerWarp];
  __shared__ uint32_t s_rowid[kTrieMaxRows];
  __shared__ __align__(8) uint64_t s_full[2];

  const uint32_t b = blockIdx.x % n_blocks;
  const uint32_t part = blockIdx.x / n_blocks;
  const TrieBlock blk = blocks[b];
  const uint32_t st0 = (uint32_t)((uint64_t)n_stripes * part / n_parts);
  const uint32_t st1 = (uint32_t)((uint64_t)n_stripes * (part + 1) / n_parts);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;

  for (uint32_t i = threadIdx.x; i < blk.n_cand; i += kThreads) {
    s_lrows[i] = cand_lrows[blk.cand_begin + i];
    s_lcp[i] = cand_lcp[blk.cand_begin + i];
  }
  for (uint32_t i = threadIdx.x; i < blk.n_rows; i += kThreads) s_rowid[i] = block_rows[blk.row_begin + i];
  const uint32_t full0 = smem_u32(&s_full[0]);
  if (threadIdx.x == 0) {
    mbar_init(full0, 1);
    mbar_init(full0 + 8, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  if (st0 >= st1) return;

  const uint32_t buf0 = smem_u32(smem);
  const uint32_t buf_bytes = blk.n_rows * kSegBytes;

  // warp 0 issues the bulk copies of stripe s into buffer (i & 1)
  auto issue = [&](uint32_t s, uint32_t i) {
    if (warp == 0) {
      const uint32_t bar = full0 + 8 * (i & 1);
      const uint64_t w0 = (uint64_t)s * kStripeWords;
      const uint32_t words = (uint32_t)((pitch_words - w0) < (uint64_t)kStripeWords ? (pitch_words - w0) : (uint64_t)kStripeWords);
      if (lane == 0) mbar_arrive_expect_tx(bar, words * 4 * blk.n_rows);
      __syncwarp();
      const uint32_t dst = buf0 + (i & 1) * buf_bytes;
      for (uint32_t r = lane; r < blk.n_rows; r += 32)
        bulk_g2s(dst + r * kSegBytes, rows + (uint64_t)s_rowid[r] * pitch_words + w0, words * 4, bar);
    }
  };

  const int my0 = warp * kCandPerWarp;
  const int n_mine = max(0, min(kCandPerWarp, (int)blk.n_cand - my0));
  uint32_t acc[kCandPerWarp];
#pragma unroll
  for (int j = 0; j < kCandPerWarp; ++j) acc[j] = 0;
  uint4 V[K - 1];
#pragma unroll
  for (int d = 0; d < K - 1; ++d) V[d] = make_uint4(0, 0, 0, 0);

  issue(st0, 0);
  for (uint32_t s = st0, i = 0; s < st1; ++s, ++i) {
    if (s + 1 < st1) issue(s + 1, i + 1);
    mbar_wait(full0 + 8 * (i & 1), (i >> 1) & 1);
    const uint64_t w0 = (uint64_t)s * kStripeWords;
    const bool lane_ok = w0 + (uint64_t)lane * 4 < pitch_words;
    const uint32_t base = buf0 + (i & 1) * buf_bytes + lane * 16;
#pragma unroll
    for (int j = 0; j < kCandPerWarp; ++j) {
      if (j < n_mine) {
        const uint4 lr = s_lrows[my0 + j];
        const int l = s_lcp[my0 + j];
#pragma unroll
        for (int d = 0; d < K - 1; ++d) {
          if (d >= l) {
            const uint4 v = lds128(base + byte_of(lr, d) * kSegBytes);
            if (d == 0) {
              V[0] = v;
            } else {
              V[d].x = V[d - 1].x & v.x; V[d].y = V[d - 1].y & v.y;
              V[d].z = V[d - 1].z & v.z; V[d].w = V[d - 1].w & v.w;
            }
          }
        }
        const uint4 v = lds128(base + byte_of(lr, K - 1) * kSegBytes);
        const uint32_t c = (__popc(V[K - 2].x & v.x) + __popc(V[K - 2].y & v.y)) +
                           (__popc(V[K - 2].z & v.z) + __popc(V[K - 2].w & v.w));
        acc[j] += lane_ok ? c : 0u;
      }
    }
    __syncthreads();  // buffer (i & 1) may be refilled at iteration i + 2 (issued at the top of i + 1)
  }
#pragma unroll
  for (int j = 0; j < kCandPerWarp; ++j) {
    if (j < n_mine) {
      const uint32_t sum = __reduce_add_sync(0xffffffffu, acc[j]);
      if (lane == 0 && sum) atomicAdd(&counts[blk.cand_begin + my0 + j], sum);
    }
  }
}

template <int K>
void launch_k(const uint32_t* rows, uint64_t pitch_words, const TrieBlock* blocks, const uint32_t* block_rows,
              const uint4* lrows, const uint8_t* lcp, uint32_t n_blocks, uint32_t n_parts, uint32_t n_stripes,
              uint32_t max_rows, uint32_t* counts, cudaStream_t stream) {
  const size_t smem = (size_t)2 * max_rows * kSegBytes;
  static bool attr = false;
  if (!attr) {
    GPA_CUDA(cudaFuncSetAttribute(count_trie_kernel<K>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                  2 * kTrieMaxRows * kSegBytes));
    attr = true;
  }
  const uint64_t grid = (uint64_t)n_blocks * n_parts;
  GPA_REQUIRE(grid < (1ull << 31), GPA_ERR_INVALID, "count_trie: grid too large");
  count_trie_kernel<K><<<(unsigned)grid, kThreads, smem, stream>>>(rows, pitch_words, blocks, block_rows, lrows, lcp,
                                                                   n_blocks, n_parts, n_stripes, counts);
  GPA_CUDA(cudaGetLastError());
}

}  // namespace

uint32_t trie_stripes(uint64_t pitch_words) { return (uint32_t)((pitch_words + kStripeWords - 1) / kStripeWords); }

uint64_t launch_count_trie(uint32_t k, const uint32_t* rows, uint64_t pitch_words, const TrieBlock* blocks,
                           const uint32_t* block_rows, const uint4* cand_lrows, const uint8_t* cand_lcp,
                           uint32_t n_blocks, uint32_t max_rows, uint32_t n_parts, uint32_t* counts,
                           cudaStream_t stream) {
  if (n_blocks == 0) return 0;
  const uint32_t n_stripes = trie_stripes(pitch_words);
  if (n_parts > n_stripes) n_parts = n_stripes;
  if (n_parts < 1) n_parts = 1;
#define GPA_TRIE_CASE(KK)                                                                                   \
  case KK:                                                                                                  \
    launch_k<KK>(rows, pitch_words, blocks, block_rows, cand_lrows, cand_lcp, n_blocks, n_parts, n_stripes, \
                 max_rows, counts, stream);                                                                 \
    break;
  switch (k) {
    GPA_TRIE_CASE(2) GPA_TRIE_CASE(3) GPA_TRIE_CASE(4) GPA_TRIE_CASE(5) GPA_TRIE_CASE(6) GPA_TRIE_CASE(7)
    GPA_TRIE_CASE(8) GPA_TRIE_CASE(9) GPA_TRIE_CASE(10) GPA_TRIE_CASE(11) GPA_TRIE_CASE(12) GPA_TRIE_CASE(13)
    GPA_TRIE_CASE(14) GPA_TRIE_CASE(15) GPA_TRIE_CASE(16)
    default:
      fail(GPA_ERR_INVALID, "count_trie: k = %u outside [2, %u]", k, kTrieMaxK);
  }
#undef GPA_TRIE_CASE
  return (uint64_t)n_blocks * n_parts;
}

}  // namespace gpa
