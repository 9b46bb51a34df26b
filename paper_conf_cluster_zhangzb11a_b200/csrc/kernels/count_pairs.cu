// count_pairs -- generation-2 support counting as a TMA-tiled AND-popcount "Gram" (sm_100a).
//
// For k = 2 every pair of frequent items is a candidate (C_2 = L_1 join L_1, P13@474) and its
// support is popc(B[a] & B[b]) summed over the words of the two static-bitset rows (complete
// intersection, P18@394; Fig. 2 P13@2637 prints {1,3} -> 1001 = V1 AND V3).  Over all pairs
// this is the upper triangle of C[a][b] = sum_w popc(B[a][w] & B[b][w]) -- a dense
// contraction over the transaction axis, evaluated here like an integer GEMM on the CUDA
// cores (the paper's method is AND + popcount; no tensor-core kind computes AND-popc):
//   * CTA tile = 128 rows (a) x 128 rows (b), upper-triangular tiles only, times a split of
//     the word axis (K-split so that the grid fills the 148 SMs);
//   * a producer warp streams 32-word (128-byte) chunks of the 128 A rows and 128 B rows into
//     a 3-stage shared-memory ring with TMA (cp.async.bulk.tensor.2d, 128B swizzle, mbarrier
//     complete_tx); a diagonal tile loads one box and uses it as both operands;
//   * 8 consumer warps: thread (tx, ty) owns the 8 x 8 pairs (ty + 16 i, tx + 16 j); per
//     16-byte slot it loads 8 A and 8 B fragments (LDS.128, conflict-free thanks to the
//     swizzle) and does 64 x 8 AND + popcount + add into 64 register accumulators; the 8 words
//     of two slots go through a carry-save adder tree so 4 POPC count 8 words (the XU pipe that
//     runs POPC is 4x narrower than the ALU pipe that runs LOP3); diagonal tiles skip the
//     micro-pairs that lie entirely below the diagonal;
//   * epilogue: one atomicAdd per (CTA, pair a < b) into the lexicographic pair index.
// Each loaded word feeds 128 pair-words, so the kernel is bound by the POPC pipe (16 / clk /
// SM, measured: profiles/r01_microbench_popc.txt), not by HBM: DRAM traffic is about
// ceil(n/128) reads of the bitset.  Integer adds: exact and order-independent.
#include <cstdint>
#include <cuda.h>
#include <cudaTypedefs.h>
#include "../common.h"
#include "../kernels.h"

namespace gpa {
namespace {

constexpr int kTile = 128;                  // rows per tile side
constexpr int kChunkWords = 32;             // words per TMA box row (128 B = swizzle span)
constexpr int kStages = 3;
constexpr int kTreeRows = 5;   // micro-tile rows 0..4 use the 8-word adder tree, rows 5..7 two 4-word adders
constexpr int kConsumerWarps = 8;
constexpr int kThreads = (kConsumerWarps + 1) * 32;
constexpr uint32_t kBoxBytes = kTile * kChunkWords * 4;        // 16 KB
constexpr uint32_t kStageBytes = 2 * kBoxBytes;                // A + B
constexpr size_t kSmemBytes = (size_t)kStages * kStageBytes + 1024 /*align*/ + 2 * kStages * 8;

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
__device__ __forceinline__ void tma_load_2d(uint32_t dst, const void* tmap, int c0, int c1, uint32_t bar) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];" ::"r"(dst),
      "l"(tmap), "r"(c0), "r"(c1), "r"(bar)
      : "memory");
}
__device__ __forceinline__ uint32_t imad(uint32_t a, uint32_t b, uint32_t c) {
  uint32_t d;
  asm("mad.lo.u32 %0, %1, %2, %3;" : "=r"(d) : "r"(a), "r"(b), "r"(c));
  return d;
}
__device__ __forceinline__ uint4 lds128(uint32_t addr) {
  uint4 v;
  asm volatile("ld.shared.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "r"(addr));
  return v;
}

__global__ void __launch_bounds__(kThreads, 1) count_pairs_kernel(const __grid_constant__ CUtensorMap tmap,
                                                                  uint32_t n_rows, uint32_t n_blocks_side,
                                                                  uint32_t n_tiles, uint32_t chunk0, uint32_t n_chunks,
                                                                  uint32_t chunks_per_split,
                                                                  uint32_t* __restrict__ counts) {
  extern __shared__ uint8_t smem_raw[];
  const uint32_t raw = smem_u32(smem_raw);
  const uint32_t buf0 = (raw + 1023u) & ~1023u;                 // 128B swizzle atoms need 1 KB alignment
  const uint32_t bar0 = buf0 + kStages * kStageBytes;           // full[s] at bar0 + 8s, empty[s] after
  const uint32_t tile = blockIdx.x % n_tiles;
  const uint32_t split = blockIdx.x / n_tiles;
  // tile -> (bi, bj), bi <= bj, row-major over the upper triangle
  uint32_t bi = 0, rem = tile;
  while (rem >= n_blocks_side - bi) { rem -= n_blocks_side - bi; ++bi; }
  const uint32_t bj = bi + rem;
  const bool diag = bi == bj;
  const uint32_t c_begin = chunk0 + split * chunks_per_split;
  const uint32_t c_end = min(c_begin + chunks_per_split, chunk0 + n_chunks);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;

  if (threadIdx.x == 0) {
    for (int s = 0; s < kStages; ++s) {
      mbar_init(bar0 + 8 * s, 1);
      mbar_init(bar0 + 8 * (kStages + s), kConsumerWarps);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();

  if (warp == kConsumerWarps) {  // ---------------- producer warp: TMA loads
    if (lane == 0) {
      asm volatile("prefetch.tensormap [%0];" ::"l"(&tmap) : "memory");
      uint32_t stage = 0, phase = 0;
      for (uint32_t c = c_begin; c < c_end; ++c) {
        mbar_wait(bar0 + 8 * (kStages + stage), phase ^ 1);
        const uint32_t full = bar0 + 8 * stage;
        const uint32_t dst = buf0 + stage * kStageBytes;
        mbar_arrive_expect_tx(full, diag ? kBoxBytes : 2 * kBoxBytes);
        tma_load_2d(dst, &tmap, (int)(c * kChunkWords), (int)(bi * kTile), full);
        if (!diag) tma_load_2d(dst + kBoxBytes, &tmap, (int)(c * kChunkWords), (int)(bj * kTile), full);
        if (++stage == kStages) { stage = 0; phase ^= 1; }
      }
    }
    return;
  }

  // ---------------- consumer warps
  const uint32_t tx = threadIdx.x & 15, ty = threadIdx.x >> 4;
  const uint32_t swa = ty & 7, swb = tx & 7;   // 128B swizzle: 16-byte slot q of row r sits at q ^ (r & 7)
  uint32_t acc[8][8];
#pragma unroll
  for (int i = 0; i < 8; ++i)
#pragma unroll
    for (int j = 0; j < 8; ++j) acc[i][j] = 0;

  uint32_t stage = 0, phase = 0;
  for (uint32_t c = c_begin; c < c_end; ++c) {
    mbar_wait(bar0 + 8 * stage, phase);
    const uint32_t A = buf0 + stage * kStageBytes;
    const uint32_t B = diag ? A : A + kBoxBytes;
#pragma unroll 1
    for (uint32_t q = 0; q < 8; q += 2) {
      // two 16-byte slots (8 words) per pair: a 7 -> 3 carry-save adder tree plus the 8th word
      uint4 a0[8], a1[8];
#pragma unroll
      for (int i = 0; i < 8; ++i) {
        a0[i] = lds128(A + (ty + 16 * i) * 128 + ((q ^ swa) << 4));
        a1[i] = lds128(A + (ty + 16 * i) * 128 + (((q + 1) ^ swa) << 4));
      }
#pragma unroll
      for (int j = 0; j < 8; ++j) {
        const uint4 b0 = lds128(B + (tx + 16 * j) * 128 + ((q ^ swb) << 4));
        const uint4 b1 = lds128(B + (tx + 16 * j) * 128 + (((q + 1) ^ swb) << 4));
#pragma unroll
        for (int i = 0; i < 8; ++i) {
          // diagonal tile: micro-pairs with i > j have a = ty + 16i > b = tx + 16j for every thread
          if (diag && i > j) continue;
          if (i < kTreeRows) {
            // popcount of 8 AND words with 4 POPC (XU pipe, 16/clk/SM) instead of 8, paid with
            // 8 LOP3 (ALU pipe, 64/clk/SM): full adders (x0,x1,x2) -> (s1,c1), (x3,x4,x5) ->
            // (s2,c2), (s1,s2,x6) -> (ones,c3), (c1,c2,c3) -> (twos,fours);
            // total = ones + x7 + 2 twos + 4 fours
            const uint32_t x0 = a0[i].x & b0.x, x1 = a0[i].y & b0.y, x2 = a0[i].z & b0.z, x3 = a0[i].w & b0.w;
            const uint32_t x4 = a1[i].x & b1.x, x5 = a1[i].y & b1.y, x6 = a1[i].z & b1.z, x7 = a1[i].w & b1.w;
            const uint32_t s1 = x0 ^ x1 ^ x2, c1 = (x0 & x1) | (x2 & (x0 ^ x1));
            const uint32_t s2 = x3 ^ x4 ^ x5, c2 = (x3 & x4) | (x5 & (x3 ^ x4));
            const uint32_t ones = s1 ^ s2 ^ x6, c3 = (s1 & s2) | (x6 & (s1 ^ s2));
            const uint32_t twos = c1 ^ c2 ^ c3, fours = (c1 & c2) | (c3 & (c1 ^ c2));
            // the accumulation runs on the FMA pipe (IMAD), leaving the ALU pipe to the LOP3s
            acc[i][j] = imad(__popc(ones), 1u, acc[i][j]);
            acc[i][j] = imad(__popc(x7), 1u, acc[i][j]);
            acc[i][j] = imad(__popc(twos), 2u, acc[i][j]);
            acc[i][j] = imad(__popc(fours), 4u, acc[i][j]);
          } else {
            // the other rows: one full adder per 4 words (3 POPC / 4 words) -- fewer LOP3, more
            // POPC, so that the ALU and XU pipes are loaded evenly
            const uint32_t x0 = a0[i].x & b0.x, x1 = a0[i].y & b0.y, x2 = a0[i].z & b0.z, x3 = a0[i].w & b0.w;
            const uint32_t x4 = a1[i].x & b1.x, x5 = a1[i].y & b1.y, x6 = a1[i].z & b1.z, x7 = a1[i].w & b1.w;
            const uint32_t s1 = x0 ^ x1 ^ x2, c1 = (x0 & x1) | (x2 & (x0 ^ x1));
            const uint32_t s2 = x4 ^ x5 ^ x6, c2 = (x4 & x5) | (x6 & (x4 ^ x5));
            acc[i][j] = imad(__popc(s1), 1u, acc[i][j]);
            acc[i][j] = imad(__popc(x3), 1u, acc[i][j]);
            acc[i][j] = imad(__popc(c1), 2u, acc[i][j]);
            acc[i][j] = imad(__popc(s2), 1u, acc[i][j]);
            acc[i][j] = imad(__popc(x7), 1u, acc[i][j]);
            acc[i][j] = imad(__popc(c2), 2u, acc[i][j]);
          }
        }
      }
    }
    __syncwarp();
    if (lane == 0) mbar_arrive(bar0 + 8 * (kStages + stage));
    if (++stage == kStages) { stage = 0; phase ^= 1; }
  }

#pragma unroll
  for (int i = 0; i < 8; ++i) {
    const uint32_t a = bi * kTile + ty + 16 * i;
#pragma unroll
    for (int j = 0; j < 8; ++j) {
      const uint32_t b = bj * kTile + tx + 16 * j;
      if (a < b && b < n_rows && acc[i][j]) atomicAdd(&counts[pair_index(a, b, n_rows)], acc[i][j]);
    }
  }
}

PFN_cuTensorMapEncodeTiled_v12000 get_encode() {
  static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
  if (!fn) {
    void* p = nullptr;
    cudaDriverEntryPointQueryResult q;
    GPA_CUDA(cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q));
    GPA_REQUIRE(q == cudaDriverEntryPointSuccess && p, GPA_ERR_CUDA, "cuTensorMapEncodeTiled unavailable");
    fn = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(p);
  }
  return fn;
}

}  // namespace

bool make_pairs_tensor_map(void* tmap128, const uint32_t* rows, uint32_t n_rows, uint64_t pitch_words) {
  static_assert(sizeof(CUtensorMap) == 128, "CUtensorMap size");
  auto encode = get_encode();
  cuuint64_t dims[2] = {pitch_words, n_rows};
  cuuint64_t strides[1] = {pitch_words * 4};
  cuuint32_t box[2] = {kChunkWords, kTile};
  cuuint32_t estr[2] = {1, 1};
  CUresult r = encode(reinterpret_cast<CUtensorMap*>(tmap128), CU_TENSOR_MAP_DATA_TYPE_UINT32, 2,
                      const_cast<uint32_t*>(rows), dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                      CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  GPA_REQUIRE(r == CUDA_SUCCESS, GPA_ERR_CUDA, "cuTensorMapEncodeTiled failed (%d)", (int)r);
  return true;
}

uint64_t launch_count_pairs(const void* tmap128, uint32_t n_rows, uint64_t word_begin, uint64_t word_end,
                            uint32_t* counts, int n_sms, cudaStream_t stream) {
  if (n_rows < 2 || word_end <= word_begin) return 0;
  const uint32_t nb = (n_rows + kTile - 1) / kTile;
  const uint32_t n_tiles = nb * (nb + 1) / 2;
  const uint32_t chunk0 = (uint32_t)(word_begin / kChunkWords);
  const uint32_t n_chunks = (uint32_t)((word_end - word_begin) / kChunkWords);
  // K-split: about 4 waves of resident CTAs, never more splits than chunks.
  const uint64_t target = (uint64_t)n_sms * 2 * 4;
  uint32_t splits = (uint32_t)(target / n_tiles);
  if (splits < 1) splits = 1;
  if (splits > n_chunks) splits = n_chunks;
  const uint32_t per = (n_chunks + splits - 1) / splits;
  splits = (n_chunks + per - 1) / per;
  const uint64_t grid = (uint64_t)n_tiles * splits;
  GPA_REQUIRE(grid < (1ull << 31), GPA_ERR_INVALID, "count_pairs: grid too large");
  ensure_smem_attr(reinterpret_cast<const void*>(count_pairs_kernel), (int)kSmemBytes);
  CUtensorMap map;
  memcpy(&map, tmap128, sizeof(map));
  { count_pairs_kernel<<<(unsigned)grid, kThreads, kSmemBytes, stream>>>(map, n_rows, nb, n_tiles, chunk0, n_chunks, per,
                                                                       counts); note_launch(); }
  GPA_CUDA(cudaGetLastError());
  return grid;
}

}  // namespace gpa
