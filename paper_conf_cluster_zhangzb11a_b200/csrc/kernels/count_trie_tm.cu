// count_trie_tm -- the transaction-tiled trie walk of count_trie.cu (generations k >= 3) with the
// stripe's rows served from TENSOR MEMORY instead of shared memory (sm_100a).
//
// Complete intersection (PAPER.md P18@394-1300): supp(c) = sum_w popc(B[c_1][w] & ... & B[c_k][w]),
// the candidates of a generation walked in lexicographic (trie) order so that shared prefixes are
// ANDed once (P13@835-1270, Fig. 4).  Same blocks, descriptors and prefix stack as count_trie.cu;
// what changes is where the row words come from.  count_trie.cu is bound by the shared-memory
// data path (ncu: ~80% of its 128 B/clk/SM wavefront peak at ~2 row loads of 1 KB per candidate
// and stripe), while tcgen05.ld reads tensor memory at ~310 B/clk/SM on a separate path
// (profiles/r01_microbench_tmem.txt).  So:
//   * a stripe is 1,024 words (32,768 transactions); TMEM lane quarter q holds words
//     [256 q, 256 q + 256) of it: lane 32 q + t has words 256 q + 4t..+3 and 256 q + 128 + 4t..+3 of
//     every block row = 8 columns per row, 32 rows = 256 columns (no replication);
//   * the producer warp bulk-copies the rows, 8 rows (32 KB) per ring slot, in the source layout
//     of tcgen05.cp.128x256b (per row: [half h][quarter q][32 lanes x 16 B]); its lane 0 copies
//     each slot into TMEM (one 4 KB tcgen05.cp per row) and tcgen05.commit's "slot free" and, after
//     the stripe's last row group, "stripe in TMEM";
//   * consumer warps q and q + 4 serve lane quarter q and split the block's candidates in halves
//     (<= 128 each: four register accumulators per lane); a row costs ONE tcgen05.ld.32x32b.x8
//     (the 8 words per lane that count_trie.cu reads with two LDS.128); all loads of a candidate
//     are in flight before one tcgen05.wait::ld, then AND / POPC exactly as before; when the
//     stripe is done they signal "TMEM free" (one stripe buffer per CTA, two CTAs per SM);
//   * the four quarters' partial counts meet in the counts array (one atomic per quarter).
// Results are identical to count_trie.cu (integer sums).
#include <cstdint>
#include "../common.h"
#include "../kernels.h"

namespace gpa {
namespace {

constexpr int kWarps = 8;                          // consumer warps
constexpr int kThreads = (kWarps + 1) * 32;        // + 1 producer warp (bulk copies + TMEM copies)
constexpr int kMaxCand = 256;                      // candidates per block (kTrieMaxCand)
constexpr uint32_t kStages = 3;                    // ring slots of 8 rows
constexpr uint32_t kGroupRows = 8;
constexpr uint32_t kStripeWords = 1024;
constexpr uint32_t kSegBytes = kStripeWords * 4;   // 4 KB of one row per stripe
constexpr uint32_t kSlotBytes = kGroupRows * kSegBytes;   // 32 KB
constexpr uint32_t kTmemCols = 256;                // 32 rows x 8 columns

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
// shared-memory matrix descriptor of 128 rows x 32 bytes (K-major, no swizzle): row i's first
// 16 bytes at 16 i (8-row core matrices 128 B apart, SBO), its second 16 bytes 2 KB later (LBO);
// sm_100 descriptor version 1
__device__ __forceinline__ uint64_t cp_desc(uint32_t saddr) {
  return (uint64_t)((saddr >> 4) & 0x3fffu) | ((uint64_t)(2048 >> 4) << 16) | ((uint64_t)(128 >> 4) << 32) |
         (1ull << 46);
}
__device__ __forceinline__ void tmem_cp(uint32_t taddr, uint64_t desc) {
  asm volatile("tcgen05.cp.cta_group::1.128x256b [%0], %1;" ::"r"(taddr), "l"(desc) : "memory");
}
__device__ __forceinline__ void tmem_commit(uint32_t bar) {
  asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(bar) : "memory");
}
struct Row8 {
  uint32_t w[8];
};
__device__ __forceinline__ void tld8(Row8& v, uint32_t taddr) {
  asm volatile("tcgen05.ld.sync.aligned.32x32b.x8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
               : "=r"(v.w[0]), "=r"(v.w[1]), "=r"(v.w[2]), "=r"(v.w[3]), "=r"(v.w[4]), "=r"(v.w[5]), "=r"(v.w[6]),
                 "=r"(v.w[7])
               : "r"(taddr));
}
__device__ __forceinline__ void tld_wait() { asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory"); }
// an empty volatile asm that "rewrites" the registers of a loaded row, placed after tld_wait():
// no use of the row can be scheduled before the wait
__device__ __forceinline__ void tie(Row8& v) {
  asm volatile("" : "+r"(v.w[0]), "+r"(v.w[1]), "+r"(v.w[2]), "+r"(v.w[3]), "+r"(v.w[4]), "+r"(v.w[5]), "+r"(v.w[6]),
               "+r"(v.w[7]));
}
__device__ __forceinline__ void and8(Row8& a, const Row8& b) {
#pragma unroll
  for (int j = 0; j < 8; ++j) a.w[j] &= b.w[j];
}

// descriptor: 16-bit fields per level (levels 0-7 in lo, 8-15 in hi) = local row * 32; the low 5
// bits of level 0's field carry the candidate's lcp.  TMEM column of level d = field >> 2.
constexpr uint32_t kLcpMask = 31u;
__device__ __forceinline__ uint32_t col_of(const uint4& lo, const uint4& hi, int d) {
  const uint4& v = d < 8 ? lo : hi;
  const int e = d & 7;
  const uint32_t w = e < 2 ? v.x : e < 4 ? v.y : e < 6 ? v.z : v.w;
  return (((e & 1) ? (w >> 16) : w) & 0xffe0u) >> 2;
}

template <int K>
constexpr int kRegLevels = K - 1 < 3 ? K - 1 : 3;

template <int K>
__global__ void __launch_bounds__(kThreads, 2) count_trie_tm_kernel(
    const uint32_t* __restrict__ rows, uint64_t pitch_words, const TrieBlock* __restrict__ blocks,
    const uint32_t* __restrict__ block_rows, const uint4* __restrict__ cand_lrows, const uint8_t* __restrict__ cand_lcp,
    uint32_t n_blocks, uint32_t n_parts, uint32_t n_stripes, uint32_t* __restrict__ counts) {
  constexpr int R = kRegLevels<K>;
  constexpr int D0 = K - 1 - R;
  extern __shared__ __align__(1024) uint8_t smem[];
  __shared__ uint4 s_desc[kMaxCand][K > 8 ? 2 : 1];
  __shared__ uint32_t s_rowid[kTrieWideRows];
  __shared__ __align__(8) uint64_t s_full[kStages];
  __shared__ __align__(8) uint64_t s_empty[kStages];
  __shared__ __align__(8) uint64_t s_tfull;
  __shared__ __align__(8) uint64_t s_tempty;
  __shared__ uint32_t s_tmem;

  const uint32_t b = blockIdx.x % n_blocks;
  const uint32_t part = blockIdx.x / n_blocks;
  const TrieBlock blk = blocks[b];
  const uint32_t st0 = (uint32_t)((uint64_t)n_stripes * part / n_parts);
  const uint32_t st1 = (uint32_t)((uint64_t)n_stripes * (part + 1) / n_parts);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;

  for (uint32_t i = threadIdx.x; i < blk.n_cand; i += kThreads) {
    const uint4 lr = cand_lrows[blk.cand_begin + i];
    const uint32_t w[4] = {lr.x, lr.y, lr.z, lr.w};
    uint32_t o[8];
#pragma unroll
    for (int q = 0; q < 8; ++q) {
      const uint32_t b0 = (w[q >> 1] >> (16 * (q & 1))) & 0xffu, b1 = (w[q >> 1] >> (16 * (q & 1) + 8)) & 0xffu;
      o[q] = (b0 * 32) | ((b1 * 32) << 16);
    }
    s_desc[i][0] = make_uint4(o[0] | cand_lcp[blk.cand_begin + i], o[1], o[2], o[3]);
    if constexpr (K > 8) s_desc[i][K > 8 ? 1 : 0] = make_uint4(o[4], o[5], o[6], o[7]);
  }
  for (uint32_t i = threadIdx.x; i < blk.n_rows; i += kThreads) s_rowid[i] = block_rows[blk.row_begin + i];
  const uint32_t full0 = smem_u32(&s_full[0]), empty0 = smem_u32(&s_empty[0]);
  const uint32_t tfull = smem_u32(&s_tfull), tempty = smem_u32(&s_tempty);
  if (threadIdx.x == 0) {
    for (uint32_t q = 0; q < kStages; ++q) {
      mbar_init(full0 + 8 * q, 1);
      mbar_init(empty0 + 8 * q, 1);
    }
    mbar_init(tfull, 1);
    mbar_init(tempty, kWarps);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (st0 >= st1) return;   // CTA-uniform, before any TMEM use
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(&s_tmem)),
                 "r"(kTmemCols));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  const uint32_t tmem = s_tmem;

  const uint32_t buf0 = smem_u32(smem);
  const uint32_t n = st1 - st0;
  const uint32_t G = (blk.n_rows + kGroupRows - 1) / kGroupRows;   // row groups per stripe (<= 4)

  if (warp == kWarps) {
    // ---------------- producer warp: unit u = (stripe u / G, row group u % G) -> ring slot u % 3
    // (all lanes: bulk copies); lane 0 copies the slot into TMEM
    const uint32_t n_units = n * G;
    auto load = [&](uint32_t u) {
      const uint32_t slot = u % kStages, s = u / G, g = u % G;
      mbar_wait(empty0 + 8 * slot, ((u / kStages) & 1) ^ 1);
      const uint32_t r0 = g * kGroupRows, nr = min(kGroupRows, blk.n_rows - r0);
      const uint32_t bar = full0 + 8 * slot;
      if (lane == 0) mbar_arrive_expect_tx(bar, kSegBytes * nr);
      __syncwarp();
      const uint64_t w0 = (uint64_t)(st0 + s) * kStripeWords;
      const uint32_t dst = buf0 + slot * kSlotBytes;
      // piece p = (h, q): words [256 q + 128 h, +128) of the stripe -> byte 2048 h + 512 q of the row
      for (uint32_t x = lane; x < nr * 8; x += 32) {
        const uint32_t r = x >> 3, h = (x >> 2) & 1, q = x & 3;
        bulk_g2s(dst + r * kSegBytes + h * 2048 + q * 512,
                 rows + (uint64_t)s_rowid[r0 + r] * pitch_words + w0 + q * 256 + h * 128, 512, bar);
      }
    };
    for (uint32_t u = 0; u < n_units && u < kStages; ++u) load(u);
    for (uint32_t u = 0; u < n_units; ++u) {
      const uint32_t slot = u % kStages, s = u / G, g = u % G;
      if (lane == 0) {
        mbar_wait(full0 + 8 * slot, (u / kStages) & 1);            // row group in shared memory
        if (g == 0) mbar_wait(tempty, (s & 1) ^ 1);                // consumers done with stripe s - 1
        asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
        const uint32_t r0 = g * kGroupRows, nr = min(kGroupRows, blk.n_rows - r0);
        const uint32_t src = buf0 + slot * kSlotBytes;
        for (uint32_t r = 0; r < nr; ++r) tmem_cp(tmem + 8 * (r0 + r), cp_desc(src + r * kSegBytes));
        tmem_commit(empty0 + 8 * slot);
        if (g == G - 1) tmem_commit(tfull);
      }
      __syncwarp();
      if (u + kStages < n_units) load(u + kStages);
    }
    return;
  }

  // ---------------- consumer warps: warps q and q + 4 read lane quarter q (words [256 q, 256 q +
  // 256) of each stripe) and take one half of the block's candidates each; lane j accumulates
  // candidates my0 + 32 a + j (a = 0..3) over all stripes of the part
  const int half = warp >> 2;
  const int chunk = ((int)blk.n_cand + 1) / 2;
  const int my0 = half * chunk;
  const int n_mine = max(0, min(chunk, (int)blk.n_cand - my0));
  const uint32_t tq = tmem + ((uint32_t)((warp & 3) * 32) << 16);
  uint32_t acc0 = 0, acc1 = 0, acc2 = 0, acc3 = 0;
  Row8 V[R];
#pragma unroll
  for (int d = 0; d < R; ++d)
#pragma unroll
    for (int j = 0; j < 8; ++j) V[d].w[j] = 0;

  // one candidate: recompute the stack from the first level that differs from the previous
  // candidate (l = lcp, warp-uniform; forced to 0 at the warp's first candidate of a stripe),
  // all of its row loads in flight before one wait
  auto candidate = [&](const uint4& lo, const uint4& hi, bool first) -> uint32_t {
    const int l = first ? 0 : (int)(lo.x & kLcpMask);
    int from = l;
    if (l <= D0) {
      // fold rows 0..D0 -> V[0], 4 loads in flight at a time
      Row8 f[4];
#pragma unroll
      for (int d0 = 0; d0 <= D0; d0 += 4) {
#pragma unroll
        for (int u = 0; u < 4; ++u)
          if (d0 + u <= D0) tld8(f[u], tq + col_of(lo, hi, d0 + u));
        tld_wait();
#pragma unroll
        for (int u = 0; u < 4; ++u)
          if (d0 + u <= D0) tie(f[u]);
#pragma unroll
        for (int u = 0; u < 4; ++u)
          if (d0 + u <= D0) {
            if (d0 + u == 0) V[0] = f[0];
            else and8(V[0], f[u]);
          }
      }
      from = D0 + 1;
    }
    Row8 L[R], leaf;
#pragma unroll
    for (int i = 1; i < R; ++i)
      if (from <= D0 + i) tld8(L[i], tq + col_of(lo, hi, D0 + i));
    tld8(leaf, tq + col_of(lo, hi, K - 1));
    tld_wait();
    tie(leaf);
#pragma unroll
    for (int i = 1; i < R; ++i)
      if (from <= D0 + i) tie(L[i]);
#pragma unroll
    for (int i = 1; i < R; ++i)
      if (from <= D0 + i) {
        V[i] = V[i - 1];
        and8(V[i], L[i]);
      }
    uint32_t c = 0;
#pragma unroll
    for (int j = 0; j < 8; ++j) c += __popc(V[R - 1].w[j] & leaf.w[j]);
    return c;
  };

  for (uint32_t i = 0; i < n; ++i) {
    mbar_wait(tfull, i & 1);
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    // candidates in pairs: both lane partials (<= 32 x 8 x 32 = 8,192 summed over the warp) share
    // one redux.sync, packed into 16-bit halves
#pragma unroll 1
    for (int j = 0; j < n_mine; j += 2) {
      const bool two = j + 1 < n_mine;
      const uint4 lo0 = s_desc[my0 + j][0];
      const uint4 hi0 = K > 8 ? s_desc[my0 + j][K > 8 ? 1 : 0] : make_uint4(0, 0, 0, 0);
      const uint4 lo1 = s_desc[my0 + j + (two ? 1 : 0)][0];
      const uint4 hi1 = K > 8 ? s_desc[my0 + j + (two ? 1 : 0)][K > 8 ? 1 : 0] : make_uint4(0, 0, 0, 0);
      uint32_t c = candidate(lo0, hi0, j == 0);
      if (two) c |= candidate(lo1, hi1, false) << 16;
      c = __reduce_add_sync(0xffffffffu, c);
      const int jj = j & 31;
      const uint32_t add = lane == jj ? (c & 0xffffu) : (lane == jj + 1 ? (c >> 16) : 0u);
      const int a = j >> 5;   // warp-uniform
      if (a == 0) acc0 += add;
      else if (a == 1) acc1 += add;
      else if (a == 2) acc2 += add;
      else acc3 += add;
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncwarp();
    if (lane == 0) mbar_arrive(tempty);
  }
  const uint32_t accs[4] = {acc0, acc1, acc2, acc3};
#pragma unroll
  for (int a = 0; a < 4; ++a) {
    const int c = 32 * a + lane;
    if (c < n_mine && accs[a]) atomicAdd(&counts[blk.cand_begin + my0 + c], accs[a]);
  }
  // teardown: warp 0 frees TMEM once every consumer warp is done with it (the producer has
  // returned after its last copy, which the consumers waited for)
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  asm volatile("bar.sync 1, %0;" ::"n"(kWarps * 32));
  if (warp == 0) {
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(kTmemCols));
  }
}

template <int K>
void launch_k(const uint32_t* rows, uint64_t pitch_words, const TrieBlock* blocks, const uint32_t* block_rows,
              const uint4* lrows, const uint8_t* lcp, uint32_t n_blocks, uint32_t n_parts, uint32_t* counts,
              cudaStream_t stream) {
  const uint32_t n_stripes = (uint32_t)(pitch_words / kStripeWords);
  if (n_parts > n_stripes) n_parts = n_stripes;
  if (n_parts < 1) n_parts = 1;
  // 3 x 32 KB ring: at most 2 CTAs (2 x 256 TMEM columns) per SM
  const size_t smem = (size_t)kStages * kSlotBytes;
  static bool attr = false;
  if (!attr) {
    GPA_CUDA(cudaFuncSetAttribute(count_trie_tm_kernel<K>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    attr = true;
  }
  const uint64_t grid = (uint64_t)n_blocks * n_parts;
  GPA_REQUIRE(grid < (1ull << 31), GPA_ERR_INVALID, "count_trie_tm: grid too large");
  count_trie_tm_kernel<K><<<(unsigned)grid, kThreads, smem, stream>>>(rows, pitch_words, blocks, block_rows, lrows, lcp,
                                                                      n_blocks, n_parts, n_stripes, counts);
  note_launch();
  GPA_CUDA(cudaGetLastError());
}

}  // namespace

uint64_t launch_count_trie_tm(uint32_t k, const uint32_t* rows, uint64_t pitch_words, const TrieBlock* blocks,
                              const uint32_t* block_rows, const uint4* cand_lrows, const uint8_t* cand_lcp,
                              uint32_t n_blocks, uint32_t max_rows, uint32_t n_parts, uint32_t* counts,
                              cudaStream_t stream) {
  if (n_blocks == 0) return 0;
  GPA_REQUIRE(k >= 3 && max_rows <= kTrieWideRows, GPA_ERR_INVALID, "count_trie_tm: k = %u, block with %u rows", k,
              max_rows);
#define GPA_TRIE_CASE(KK)                                                                                          \
  case KK:                                                                                                        \
    launch_k<KK>(rows, pitch_words, blocks, block_rows, cand_lrows, cand_lcp, n_blocks, n_parts, counts, stream);  \
    break;
  switch (k) {
    GPA_TRIE_CASE(3) GPA_TRIE_CASE(4) GPA_TRIE_CASE(5) GPA_TRIE_CASE(6) GPA_TRIE_CASE(7) GPA_TRIE_CASE(8)
    GPA_TRIE_CASE(9) GPA_TRIE_CASE(10) GPA_TRIE_CASE(11) GPA_TRIE_CASE(12) GPA_TRIE_CASE(13) GPA_TRIE_CASE(14)
    GPA_TRIE_CASE(15) GPA_TRIE_CASE(16)
    default:
      fail(GPA_ERR_INVALID, "count_trie_tm: k = %u outside [3, %u]", k, kTrieMaxK);
  }
#undef GPA_TRIE_CASE
  const uint32_t n_stripes = (uint32_t)(pitch_words / kStripeWords);
  return (uint64_t)n_blocks * (n_parts > n_stripes ? n_stripes : (n_parts < 1 ? 1 : n_parts));
}

}  // namespace gpa
