// Static bitset construction (sm_100a).
//
// "Only the vertical lists of first generation will be saved in graphics memory" (PAPER.md
// P18@755); each list is a bitmask over all transactions, the "static bitset" (P2@270,
// P13@1844), rows aligned for coalesced access (P18@1685).  The paper does not say how the
// rows are built; here the horizontal CSR is transposed on the device:
//   CTA (chunk c, row block rb) owns transactions [512c, 512c + 512) = words [16c, 16c + 16)
//   of rows [rb*RB, rb*RB + RB).  It zeroes a shared-memory tile of RB rows x 16 words (row
//   stride 17 words: lanes writing the same word column of different rows hit different
//   banks; 68 KB for 1,024 rows -> 3 CTAs per SM to hide the gather latency), scans the chunk's
//   transactions (one thread per transaction, 4 item -> row gathers in flight), sets bits with
//   shared-memory atomicOr (duplicates are harmless: OR is idempotent, so non-canonical input
//   needs no special case), then writes every row's 64-byte segment with coalesced stores.  Every word of the output is written (padding
//   transactions contribute no bits, so padding is zero).
#include <cstdint>
#include "../common.h"
#include "../kernels.h"

namespace gpa {
namespace {

constexpr int kBuildThreads = 256;
constexpr uint32_t kChunkTx = 512;       // transactions per CTA = 16 words (64-byte row segments)
constexpr uint32_t kChunkWords = kChunkTx / 32;
constexpr uint32_t kTileStride = 17;     // padded words per tile row (odd: conflict-free columns)
constexpr uint32_t kRowBlock = 1024;     // rows per CTA tile: 1024 * 17 * 4 = 68 KB -> 3 CTAs / SM

__global__ void __launch_bounds__(kBuildThreads) bitset_build_kernel(const uint64_t* __restrict__ offsets,
                                                                     const uint32_t* __restrict__ items,
                                                                     uint64_t n_tx, const int32_t* __restrict__ row_of_item,
                                                                     uint32_t n_rows, uint32_t row_block,
                                                                     uint64_t pitch_words, uint32_t* __restrict__ rows) {
  extern __shared__ uint32_t tile[];
  const uint64_t chunk = blockIdx.x;
  const uint32_t rb0 = blockIdx.y * row_block;
  const uint32_t nr = min(row_block, n_rows - rb0);
  for (uint32_t i = threadIdx.x; i < nr * kTileStride; i += blockDim.x) tile[i] = 0;
  __syncthreads();
  const uint64_t t0 = chunk * kChunkTx;
  for (uint32_t tl = threadIdx.x; tl < kChunkTx; tl += blockDim.x) {
    const uint64_t t = t0 + tl;
    if (t >= n_tx) break;
    const uint64_t o0 = __ldg(offsets + t), o1 = __ldg(offsets + t + 1);
    const uint32_t bit = 1u << (tl & 31);
    const uint32_t wcol = tl >> 5;
    uint64_t j = o0;
    for (; j + 4 <= o1; j += 4) {  // 4 independent item -> row gathers in flight
      uint32_t it[4];
      int32_t r[4];
#pragma unroll
      for (int u = 0; u < 4; ++u) it[u] = __ldg(items + j + u);
#pragma unroll
      for (int u = 0; u < 4; ++u) r[u] = __ldg(row_of_item + it[u]);
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        const uint32_t rr = (uint32_t)r[u] - rb0;   // r < 0 wraps to a huge value: skipped
        if (r[u] >= 0 && rr < nr) atomicOr(&tile[rr * kTileStride + wcol], bit);
      }
    }
    for (; j < o1; ++j) {
      const int32_t r = __ldg(row_of_item + __ldg(items + j));
      const uint32_t rr = (uint32_t)r - rb0;
      if (r >= 0 && rr < nr) atomicOr(&tile[rr * kTileStride + wcol], bit);
    }
  }
  __syncthreads();
  uint32_t* out = rows + (uint64_t)rb0 * pitch_words + chunk * kChunkWords;
  for (uint32_t i = threadIdx.x; i < nr * kChunkWords; i += blockDim.x) {
    const uint32_t r = i / kChunkWords, w = i % kChunkWords;
    out[(uint64_t)r * pitch_words + w] = tile[r * kTileStride + w];
  }
}

}  // namespace

void launch_bitset_build(const uint64_t* offsets, const uint32_t* items, uint64_t n_tx, const int32_t* row_of_item,
                         uint32_t n_rows, uint64_t pitch_words, uint32_t* rows, cudaStream_t stream) {
  if (n_rows == 0) return;
  const uint64_t n_chunks = pitch_words / kChunkWords;
  const uint32_t rb = n_rows < kRowBlock ? n_rows : kRowBlock;
  const uint32_t n_rb = (n_rows + rb - 1) / rb;
  const size_t smem = (size_t)rb * kTileStride * sizeof(uint32_t);
  GPA_CUDA(cudaFuncSetAttribute(bitset_build_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  GPA_REQUIRE(n_chunks < (1ull << 31), GPA_ERR_INVALID, "bitset: too many transactions");
  dim3 grid((unsigned)n_chunks, n_rb);
  bitset_build_kernel<<<grid, kBuildThreads, smem, stream>>>(offsets, items, n_tx, row_of_item, n_rows, rb,
                                                             pitch_words, rows);
  GPA_CUDA(cudaGetLastError());
}

}  // namespace gpa
