// count_pairs_tc -- generation-2 support counting on the 5th-generation tensor cores (sm_100a).
//
// For k = 2 every pair of frequent items is a candidate (C_2 = L_1 join L_1, P13@474) and its
// support is the complete intersection popc(B[a] & B[b]) over the static-bitset rows (P18@394;
// Fig. 2 P13@2637 prints {1,3} -> 1001 = V1 AND V3).  Over all pairs this is the upper triangle of
// the Gram matrix C = B B^T of the 0/1 matrix B (rows = frequent items, columns = transactions):
// for bits, AND is the product and popcount the sum, so
//     C[a][b] = sum_t B[a][t] * B[b][t]   exactly, in integers.
// Generation 2 is the one place where the hot path IS a dense contraction (every (a, b) is a
// candidate), so it runs as an integer GEMM on tcgen05 (kind::i8, u8 x u8 -> s32 in TMEM):
//   * CTA tile = 128 rows a (TMEM lanes, M = 128) x 256 rows b (TMEM columns, N = 256), only tiles
//     that reach the upper triangle, times a split of the transaction axis (K) over the grid;
//   * 12 producer warps = one thread per tile row: each stage covers 128 transactions = 4 bit-words
//     per row, loaded with one 16-byte read-only load (two stages in flight in registers),
//     expanded bit -> byte (word j of a 16-byte chunk holds bits j, j+8, j+16, j+24 of the bit-word:
//     (w >> j) & 0x01010101 -- a fixed permutation of the K axis, identical for both operands, so
//     every dot product is unchanged) and stored into the canonical K-major no-swizzle UMMA layout
//     (8-row x 16-byte core matrices, conflict-free 128-byte quarter-warp stores), then
//     fence.proxy.async + mbarrier arrive; 4-stage ring (48 KB per stage);
//   * one elected thread issues 4 tcgen05.mma (M128 N256 K32) per stage and tcgen05.commit's the
//     stage's empty barrier; the accumulator (128 x 256 s32 = 256 TMEM columns) never leaves TMEM
//     until the end of the CTA's K range;
//   * epilogue: 4 warps (one per TMEM lane quarter) tcgen05.ld 32 columns at a time and add each
//     pair a < b into the lexicographic pair index with one atomic per (CTA, pair).
// Exact: 0/1 products, s32 accumulation (a CTA's K range < 2^31), integer atomics.
#include <cstdint>
#include "../common.h"
#include "../kernels.h"

namespace gpa {
namespace {

constexpr int kM = 128;                      // a rows per tile (TMEM lanes)
constexpr int kN = 256;                      // b rows per tile (TMEM columns)
constexpr int kWords = 4;                    // bit-words per row per stage (4 x 32 transactions)
constexpr int kStages = 4;
constexpr int kProducerWarps = (kM + kN) / 32;   // 12: one thread per tile row
constexpr int kEpiWarps = 4;                 // warps 0..3: MMA issue (warp 0) + epilogue
constexpr int kThreads = (kEpiWarps + kProducerWarps) * 32;
constexpr uint32_t kABytes = kM * kWords * 32;   // 16 KB: 4 K-steps x 128 rows x 32 bytes
constexpr uint32_t kBBytes = kN * kWords * 32;   // 32 KB
constexpr uint32_t kStageBytes = kABytes + kBBytes;
constexpr uint32_t kTmemCols = kN;           // s32 accumulator: one column per b row
constexpr size_t kSmemBytes = (size_t)kStages * kStageBytes + 1024;

// instruction descriptor (kind::i8): D = S32 (bits 4-5 = 2), A = B = unsigned 8-bit (0), both
// K-major, N >> 3 at bit 17, M >> 4 at bit 24
constexpr uint32_t kIdesc = (2u << 4) | ((uint32_t)(kN >> 3) << 17) | ((uint32_t)(kM >> 4) << 24);

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

__device__ __forceinline__ void mbar_init(uint32_t bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(bar), "r"(count));
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
// K-major, no swizzle: core matrix = 8 rows x 16 bytes; LBO = 128 B (next 16-element K chunk),
// SBO = 256 B (next 8-row group); version 1 (sm_100)
__device__ __forceinline__ uint64_t umma_desc(uint32_t saddr) {
  return (uint64_t)((saddr >> 4) & 0x3fffu) | ((uint64_t)(128 >> 4) << 16) | ((uint64_t)(256 >> 4) << 32) |
         (1ull << 46);
}
__device__ __forceinline__ void umma_i8(uint32_t tmem_d, uint64_t da, uint64_t db, uint32_t accumulate) {
  asm volatile(
      "{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\n"
      "tcgen05.mma.cta_group::1.kind::i8 [%0], %1, %2, %3, p;\n}\n" ::"r"(tmem_d),
      "l"(da), "l"(db), "r"(kIdesc), "r"(accumulate)
      : "memory");
}
__device__ __forceinline__ void umma_commit(uint32_t bar) {
  asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(bar) : "memory");
}
__device__ __forceinline__ void sts128(uint32_t addr, uint32_t a, uint32_t b, uint32_t c, uint32_t d) {
  asm volatile("st.shared.v4.u32 [%0], {%1,%2,%3,%4};" ::"r"(addr), "r"(a), "r"(b), "r"(c), "r"(d) : "memory");
}
__device__ __forceinline__ uint4 ldg_nc(const uint32_t* p) {
  uint4 v;
  asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
               : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w)
               : "l"(p));
  return v;
}

// one bit-word (32 transactions) of one row -> 32 bytes at K-step base `ks` (row r of R rows):
// chunk 0 (bytes for bits j, j+8, j+16, j+24, j = 0..3) and chunk 1 (j = 4..7)
__device__ __forceinline__ void expand_word(uint32_t w, uint32_t dst_chunk0) {
  constexpr uint32_t m = 0x01010101u;
  sts128(dst_chunk0, w & m, (w >> 1) & m, (w >> 2) & m, (w >> 3) & m);
  sts128(dst_chunk0 + 128, (w >> 4) & m, (w >> 5) & m, (w >> 6) & m, (w >> 7) & m);
}

__global__ void __launch_bounds__(kThreads, 1)
    count_pairs_tc_kernel(const uint32_t* __restrict__ rows, uint64_t pitch_words, uint32_t n_rows, uint32_t nbi,
                          uint32_t nbj, uint64_t word0, uint32_t n_stage_total, uint32_t stages_per_split,
                          uint32_t* __restrict__ counts) {
  extern __shared__ uint8_t smem_raw[];
  __shared__ __align__(8) uint64_t s_full[kStages];
  __shared__ __align__(8) uint64_t s_empty[kStages];
  __shared__ __align__(8) uint64_t s_done;
  __shared__ uint32_t s_tmem;

  const uint32_t n_tiles = nbi * nbj;
  const uint32_t tile = blockIdx.x % n_tiles;
  const uint32_t split = blockIdx.x / n_tiles;
  const uint32_t bi = tile % nbi, bj = tile / nbi;
  const uint32_t a0 = bi * kM, b0 = bj * kN;
  // a tile that never reaches a < b < n_rows does nothing
  const uint32_t b_hi = min(n_rows, b0 + kN);
  if (a0 + 1 >= b_hi) return;
  const uint32_t st0 = split * stages_per_split;
  const uint32_t st1 = min(n_stage_total, st0 + stages_per_split);
  if (st0 >= st1) return;
  const uint32_t n_st = st1 - st0;

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const uint32_t buf0 = (smem_u32(smem_raw) + 1023u) & ~1023u;
  const uint32_t full0 = smem_u32(&s_full[0]), empty0 = smem_u32(&s_empty[0]), done = smem_u32(&s_done);

  if (threadIdx.x == 0) {
    for (int s = 0; s < kStages; ++s) {
      mbar_init(full0 + 8 * s, kProducerWarps);
      mbar_init(empty0 + 8 * s, 1);
    }
    mbar_init(done, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(&s_tmem)),
                 "r"(kTmemCols));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  const uint32_t tmem = s_tmem;

  if (warp >= kEpiWarps) {
    // ---------------- producers: thread p owns tile row p (A rows 0..127, then B rows 0..255)
    const uint32_t p = threadIdx.x - kEpiWarps * 32;
    const bool is_a = p < kM;
    const uint32_t r = is_a ? p : p - kM;
    const uint32_t g = is_a ? a0 + r : b0 + r;
    const bool valid = g < n_rows;
    const uint32_t* src = rows + (uint64_t)(valid ? g : 0) * pitch_words + word0 + (uint64_t)st0 * kWords;
    // byte offset of this row's chunk 0 inside K-step 0 of a stage
    const uint32_t R = is_a ? kM : kN;
    const uint32_t row_off = (is_a ? 0u : kABytes) + (r >> 3) * 256 + (r & 7) * 16;
    uint4 v0 = valid ? ldg_nc(src) : make_uint4(0, 0, 0, 0);
    uint4 v1 = (valid && n_st > 1) ? ldg_nc(src + kWords) : make_uint4(0, 0, 0, 0);
    for (uint32_t i = 0; i < n_st; ++i) {
      const uint4 v = v0;
      v0 = v1;
      v1 = (valid && i + 2 < n_st) ? ldg_nc(src + (uint64_t)(i + 2) * kWords) : make_uint4(0, 0, 0, 0);
      const uint32_t slot = i % kStages;
      mbar_wait(empty0 + 8 * slot, ((i / kStages) & 1) ^ 1);
      const uint32_t dst = buf0 + slot * kStageBytes + row_off;
      expand_word(v.x, dst);
      expand_word(v.y, dst + R * 32);
      expand_word(v.z, dst + 2 * R * 32);
      expand_word(v.w, dst + 3 * R * 32);
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
      __syncwarp();
      if (lane == 0) mbar_arrive(full0 + 8 * slot);
    }
  } else {
    // ---------------- warp 0 lane 0: MMA issue
    if (warp == 0 && lane == 0) {
      for (uint32_t i = 0; i < n_st; ++i) {
        const uint32_t slot = i % kStages;
        mbar_wait(full0 + 8 * slot, (i / kStages) & 1);
        asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
        const uint32_t sa = buf0 + slot * kStageBytes, sb = sa + kABytes;
#pragma unroll
        for (int s = 0; s < kWords; ++s)
          umma_i8(tmem, umma_desc(sa + s * kM * 32), umma_desc(sb + s * kN * 32), (i | s) ? 1u : 0u);
        umma_commit(empty0 + 8 * slot);
      }
      umma_commit(done);
    }
    __syncwarp();
    // ---------------- epilogue: warp q reads TMEM lanes 32q..32q+31 (tile rows a), 32 columns at a time
    mbar_wait(done, 0);
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    const uint32_t a = a0 + warp * 32 + lane;
    const uint64_t n = n_rows;
    for (uint32_t c0 = 0; c0 < (uint32_t)kN; c0 += 32) {
      if (b0 + c0 >= b_hi) break;                                 // warp-uniform
      if (b0 + c0 + 31 <= a0 + warp * 32) continue;               // whole chunk at or below the diagonal
      uint32_t v[32];
      const uint32_t taddr = tmem + ((uint32_t)(warp * 32) << 16) + c0;
      asm volatile(
          "tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,"
          "%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
          : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7]),
            "=r"(v[8]), "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]), "=r"(v[14]), "=r"(v[15]),
            "=r"(v[16]), "=r"(v[17]), "=r"(v[18]), "=r"(v[19]), "=r"(v[20]), "=r"(v[21]), "=r"(v[22]),
            "=r"(v[23]), "=r"(v[24]), "=r"(v[25]), "=r"(v[26]), "=r"(v[27]), "=r"(v[28]), "=r"(v[29]),
            "=r"(v[30]), "=r"(v[31])
          : "r"(taddr));
      asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
      if (a < n_rows) {
        const uint64_t base = pair_index(a, a + 1, n) - (a + 1);   // pair_index(a, b) = base + b
#pragma unroll
        for (int j = 0; j < 32; ++j) {
          const uint32_t b = b0 + c0 + j;
          if (a < b && b < n_rows && v[j]) atomicAdd(&counts[base + b], v[j]);
        }
      }
    }
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  if (warp == 0) {
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(kTmemCols));
  }
}

}  // namespace

uint64_t launch_count_pairs_tc(const uint32_t* rows, uint64_t pitch_words, uint32_t n_rows, uint64_t word_begin,
                               uint64_t word_end, uint32_t* counts, int n_sms, cudaStream_t stream) {
  if (n_rows < 2 || word_end <= word_begin) return 0;
  GPA_REQUIRE(word_begin % kWords == 0 && word_end % kWords == 0, GPA_ERR_INVALID,
              "count_pairs_tc: word range not a multiple of %d", kWords);
  const uint32_t nbi = (n_rows + kM - 1) / kM, nbj = (n_rows + kN - 1) / kN;
  uint32_t live = 0;   // tiles that reach the upper triangle
  for (uint32_t j = 0; j < nbj; ++j)
    for (uint32_t i = 0; i < nbi; ++i)
      if (i * kM + 1 < std::min<uint32_t>(n_rows, (j + 1) * kN)) ++live;
  const uint64_t n_st = (word_end - word_begin) / kWords;
  GPA_REQUIRE(n_st < (1ull << 31), GPA_ERR_INVALID, "count_pairs_tc: word range too long");
  // K-split: about 4 waves of one CTA per SM over the live tiles
  uint64_t splits = ((uint64_t)n_sms * 4 + live - 1) / live;
  if (splits > n_st) splits = n_st;
  if (splits < 1) splits = 1;
  const uint64_t per = (n_st + splits - 1) / splits;
  splits = (n_st + per - 1) / per;
  const uint64_t grid = (uint64_t)nbi * nbj * splits;
  GPA_REQUIRE(grid < (1ull << 31), GPA_ERR_INVALID, "count_pairs_tc: grid too large");
  static bool attr = false;
  if (!attr) {
    GPA_CUDA(cudaFuncSetAttribute(count_pairs_tc_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kSmemBytes));
    attr = true;
  }
  count_pairs_tc_kernel<<<(unsigned)grid, kThreads, kSmemBytes, stream>>>(rows, pitch_words, n_rows, nbi, nbj,
                                                                          word_begin, (uint32_t)n_st, (uint32_t)per,
                                                                          counts);
  GPA_CUDA(cudaGetLastError());
  return grid;
}

}  // namespace gpa
