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
//     that reach the upper triangle (the lower diagonal tiles, whose left 128 b rows lie below the
//     diagonal, run N = 128 on the right half), times a split of the transaction axis (K): the grid is exactly
//     4 waves of one CTA per SM, the live tiles get floor or ceil(grid / tiles) K-splits each (no
//     tail wave, no idle CTAs);
//   * one thread streams the tile's bit rows with TMA (cp.async.bulk.tensor.2d, boxes of 8 words x
//     128 rows, 32-byte swizzle, 4-deep ring; out-of-range rows arrive as zeros);
//   * 12 producer warps = one thread per tile row: each stage covers 128 transactions = 4 bit-words
//     per row, read from the bit ring (one conflict-free LDS.128), expanded bit -> byte (word j of a 16-byte chunk holds bits j, j+8, j+16, j+24 of the bit-word:
//     (w >> j) & 0x01010101 -- a fixed permutation of the K axis, identical for both operands, so
//     every dot product is unchanged) and stored into the canonical K-major no-swizzle UMMA layout
//     (8-row x 16-byte core matrices, conflict-free 128-byte quarter-warp stores), then
//     fence.proxy.async + mbarrier arrive; 3-stage operand ring (48 KB per stage);
//   * one elected thread issues 4 tcgen05.mma (M128 N256 K32, A from TMEM, B from shared memory)
//     per stage and tcgen05.commit's the stage's empty barrier; the accumulator (128 x 256 s32 =
//     256 TMEM columns) never leaves TMEM until the end of the CTA's K range;
//   * epilogue: 4 warps (one per TMEM lane quarter) tcgen05.ld 32 columns at a time and add each
//     pair a < b into the lexicographic pair index with one atomic per (CTA, pair).
// Exact: 0/1 products, s32 accumulation (a CTA's K range < 2^31), integer atomics.
#include <cstdint>
#include <cstring>
#include <cuda.h>
#include <cudaTypedefs.h>
#include "../common.h"
#include "../kernels.h"

namespace gpa {
namespace {

constexpr int kM = 128;                      // a rows per tile (TMEM lanes)
constexpr int kN = 256;                      // b rows per tile (TMEM columns)
constexpr int kWords = 4;                    // bit-words per row per stage (4 x 32 transactions)
constexpr int kStages = 4;                   // operand (byte) stages
constexpr int kBitWords = 8;                 // bit ring: 8 words (256 transactions = 2 stages) per slot
constexpr int kBitStages = 4;
constexpr int kBoxRows = 128;                // TMA box: 8 words x 128 rows (32 B rows, 32-byte swizzle)
constexpr int kProducerWarps = (kM + kN) / 32;   // 12 per group: one thread per tile row
constexpr int kProducerGroups = 2;           // group g expands the stages i with i % 2 == g
constexpr int kEpiWarps = 4;                 // warps 0..3: MMA issue (warp 0) + epilogue
constexpr int kThreads = (kEpiWarps + kProducerGroups * kProducerWarps) * 32;
constexpr uint32_t kBBytes = kN * kWords * 32;   // 32 KB: 4 K-steps x 256 rows x 32 bytes
constexpr uint32_t kStageBytes = kBBytes;
constexpr uint32_t kAcol = kN;               // TMEM: accumulator in columns [0, 256), A ring after it
constexpr uint32_t kAcolsPerStage = kWords * 8;   // 32 bytes of K per row and K-step = 8 columns
constexpr uint32_t kTmemCols = 512;
constexpr uint32_t kBitStageBytes = (kM + kN) * kBitWords * 4;   // 12 KB
constexpr size_t kSmemBytes = (size_t)kStages * kStageBytes + (size_t)kBitStages * kBitStageBytes + 1024;

// instruction descriptor (kind::i8): D = S32 (bits 4-5 = 2), A = B = unsigned 8-bit (0), both
// K-major, N >> 3 at bit 17, M >> 4 at bit 24
constexpr uint32_t kIdesc = (2u << 4) | ((uint32_t)(kN >> 3) << 17) | ((uint32_t)(kM >> 4) << 24);
// the lower diagonal tiles (row block bi = 2 bj + 1): their left 128 b columns lie entirely below the
// diagonal, so they run N = 128 on the right half only
constexpr uint32_t kIdescHalf = (2u << 4) | ((uint32_t)((kN / 2) >> 3) << 17) | ((uint32_t)(kM >> 4) << 24);

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
// D[tmem] (+)= A[tmem] . B[smem]^T
__device__ __forceinline__ void umma_i8_ta(uint32_t tmem_d, uint32_t tmem_a, uint64_t db, uint32_t accumulate,
                                           uint32_t idesc) {
  asm volatile(
      "{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\n"
      "tcgen05.mma.cta_group::1.kind::i8 [%0], [%1], %2, %3, p;\n}\n" ::"r"(tmem_d),
      "r"(tmem_a), "l"(db), "r"(idesc), "r"(accumulate)
      : "memory");
}
// w >> j as the high word of w * 2^(32 - j) (IMAD.HI on the FMA pipe) -- the expansion below is
// ALU-bound otherwise (SHF + LOP3 per byte lane); sh.m[j] = 2^(32 - j) arrives through a kernel
// argument so the compiler cannot fold it back into a shift
struct Shr {
  uint32_t m[8];
  __device__ __forceinline__ uint32_t operator()(uint32_t w, int j) const { return j ? __umulhi(w, m[j]) : w; }
};
// one K-step of one A row (this thread's TMEM lane): 8 columns of 4 bytes
__device__ __forceinline__ void expand_word_tmem(uint32_t w, uint32_t taddr, const Shr& sh) {
  constexpr uint32_t m = 0x01010101u;
  asm volatile("tcgen05.st.sync.aligned.32x32b.x8.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};" ::"r"(taddr), "r"(w & m),
               "r"(sh(w, 1) & m), "r"(sh(w, 2) & m), "r"(sh(w, 3) & m), "r"(sh(w, 4) & m), "r"(sh(w, 5) & m),
               "r"(sh(w, 6) & m), "r"(sh(w, 7) & m)
               : "memory");
}
__device__ __forceinline__ void umma_commit(uint32_t bar) {
  asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(bar) : "memory");
}
__device__ __forceinline__ void sts128(uint32_t addr, uint32_t a, uint32_t b, uint32_t c, uint32_t d) {
  asm volatile("st.shared.v4.u32 [%0], {%1,%2,%3,%4};" ::"r"(addr), "r"(a), "r"(b), "r"(c), "r"(d) : "memory");
}
__device__ __forceinline__ uint4 lds128(uint32_t addr) {
  uint4 v;
  asm volatile("ld.shared.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "r"(addr));
  return v;
}
__device__ __forceinline__ void mbar_arrive_expect_tx(uint32_t bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes) : "memory");
}
__device__ __forceinline__ void tma_load_2d(uint32_t dst, const void* tmap, int c0, int c1, uint32_t bar) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];" ::"r"(dst),
      "l"(tmap), "r"(c0), "r"(c1), "r"(bar)
      : "memory");
}

// one bit-word (32 transactions) of one row -> 32 bytes at K-step base `ks` (row r of R rows):
// chunk 0 (bytes for bits j, j+8, j+16, j+24, j = 0..3) and chunk 1 (j = 4..7)
__device__ __forceinline__ void expand_word(uint32_t w, uint32_t dst_chunk0, const Shr& sh) {
  constexpr uint32_t m = 0x01010101u;
  sts128(dst_chunk0, w & m, sh(w, 1) & m, sh(w, 2) & m, sh(w, 3) & m);
  sts128(dst_chunk0 + 128, sh(w, 4) & m, sh(w, 5) & m, sh(w, 6) & m, sh(w, 7) & m);
}

__global__ void __launch_bounds__(kThreads, 1)
    count_pairs_tc_kernel(const __grid_constant__ CUtensorMap tmap, uint32_t n_rows, uint32_t nbi,
                          uint32_t n_live, uint64_t word0, uint32_t n_bit_stages, uint32_t one,
                          uint32_t* __restrict__ counts) {
  extern __shared__ uint8_t smem_raw[];
  __shared__ __align__(8) uint64_t s_full[kStages];
  __shared__ __align__(8) uint64_t s_empty[kStages];
  __shared__ __align__(8) uint64_t s_done;
  __shared__ __align__(8) uint64_t s_bfull[kBitStages];
  __shared__ __align__(8) uint64_t s_bempty[kBitStages];
  __shared__ uint32_t s_tmem;

  // CTA -> (live tile t, split si of S_t): splits interleaved across tiles, tile t gets
  // q + (t < r) of them (q, r = grid / n_live, grid % n_live)
  const uint32_t q = gridDim.x / n_live, rr = gridDim.x % n_live;
  uint32_t t, si;
  if (blockIdx.x < q * n_live) { t = blockIdx.x % n_live; si = blockIdx.x / n_live; }
  else { t = blockIdx.x - q * n_live; si = q; }
  const uint32_t S = q + (t < rr ? 1u : 0u);
  // live tile t -> (bi, bj): column bj holds the row blocks bi with bi * 128 + 1 < min(n, 256 (bj + 1))
  uint32_t bj = 0;
  for (;; ++bj) {
    const uint32_t hi = min(n_rows, (bj + 1) * (uint32_t)kN);
    const uint32_t cnt = min(nbi, (hi - 1 + kM - 1) / kM);
    if (t < cnt) break;
    t -= cnt;
  }
  const uint32_t bi = t;
  // lower diagonal tile: b columns [256 bj, 256 bj + 128) < a0 -- only the right half is counted
  // (N = 128, the B half loaded as B rows 0..127)
  const bool half = bi == 2 * bj + 1;
  const uint32_t nN = half ? kN / 2 : kN;
  const uint32_t a0 = bi * kM, b0 = bj * kN + (half ? kN / 2 : 0u);
  const uint32_t b_hi = min(n_rows, b0 + nN);
  // K range of this split in whole bit stages (2 operand stages each)
  const uint32_t bs0 = (uint32_t)((uint64_t)n_bit_stages * si / S), bs1 = (uint32_t)((uint64_t)n_bit_stages * (si + 1) / S);
  if (bs0 >= bs1) return;
  const uint32_t st0 = 2 * bs0;
  const uint32_t n_st = 2 * (bs1 - bs0);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const uint32_t buf0 = (smem_u32(smem_raw) + 1023u) & ~1023u;
  const uint32_t full0 = smem_u32(&s_full[0]), empty0 = smem_u32(&s_empty[0]), done = smem_u32(&s_done);
  const uint32_t bfull0 = smem_u32(&s_bfull[0]), bempty0 = smem_u32(&s_bempty[0]);
  const uint32_t bits0 = buf0 + kStages * kStageBytes;   // bit ring (1 KB aligned: stage bytes are)
  const uint32_t n_bst = n_st / 2;                       // bit stages (n_st is even)

  if (threadIdx.x == 0) {
    for (int s = 0; s < kStages; ++s) {
      mbar_init(full0 + 8 * s, kProducerWarps);
      mbar_init(empty0 + 8 * s, 1);
    }
    mbar_init(done, 1);
    for (int s = 0; s < kBitStages; ++s) {
      mbar_init(bfull0 + 8 * s, 1);
      mbar_init(bempty0 + 8 * s, kProducerWarps);   // a bit stage is expanded by one producer group
    }
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
    // ---------------- producers: group g = 0, 1 (warps 4..15, 16..27) expands the bit stages
    // j = g mod 2 (both of their operand stages); thread p owns tile row p (A rows 0..127, then
    // B rows 0..255) -- two groups keep two bit stages in flight per row
    const uint32_t g = (uint32_t)(warp - kEpiWarps) / kProducerWarps;
    const uint32_t p = threadIdx.x - (kEpiWarps + g * kProducerWarps) * 32;
    const bool is_a = p < kM;
    const uint32_t r = is_a ? p : p - kM;
    // B: byte offset of this row's chunk 0 inside K-step 0 of a stage; A: this warp's TMEM lane
    // quarter (warps 4..7 and 16..19 = quarters 0..3 = A rows 0..127)
    const uint32_t row_off = (r >> 3) * 256 + (r & 7) * 16;
    const uint32_t ta0 = tmem + ((uint32_t)((warp & 3) * 32) << 16) + kAcol;
    // this row in the bit ring: 32-byte rows, 16-byte half h at (h ^ (row bit 2)) (32B swizzle)
    const uint32_t brow = bits0 + p * 32;
    const uint32_t bsw = (p >> 2) & 1;
    Shr sh;
#pragma unroll
    for (int j = 0; j < 8; ++j) sh.m[j] = j ? one << (32 - j) : 0u;
    // group g expands the bit stages j = g mod 2, both operand stages (halves) of each: one bit-ring
    // wait / release per two operand stages
    for (uint32_t j = g; j < n_bst; j += 2) {
      const uint32_t bslot = j % kBitStages;
      mbar_wait(bfull0 + 8 * bslot, (j / kBitStages) & 1);
      const uint32_t brs = brow + bslot * kBitStageBytes;
      const uint4 v0 = lds128(brs + (bsw << 4)), v1 = lds128(brs + ((bsw ^ 1u) << 4));
      __syncwarp();
      if (lane == 0) mbar_arrive(bempty0 + 8 * bslot);
#pragma unroll
      for (uint32_t h = 0; h < 2; ++h) {
      const uint32_t i = 2 * j + h;
      const uint4 v = h ? v1 : v0;
      const uint32_t slot = i % kStages;
      mbar_wait(empty0 + 8 * slot, ((i / kStages) & 1) ^ 1);
      if (half && !is_a && r >= kN / 2) {
        // B rows past the half: not used by the N = 128 MMA (warp-uniform)
      } else if (is_a) {   // warp-uniform
        const uint32_t ta = ta0 + slot * kAcolsPerStage;
        expand_word_tmem(v.x, ta, sh);
        expand_word_tmem(v.y, ta + 8, sh);
        expand_word_tmem(v.z, ta + 16, sh);
        expand_word_tmem(v.w, ta + 24, sh);
        asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
        asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
      } else {
        const uint32_t dst = buf0 + slot * kStageBytes + row_off;
        expand_word(v.x, dst, sh);
        expand_word(v.y, dst + kN * 32, sh);
        expand_word(v.z, dst + 2 * kN * 32, sh);
        expand_word(v.w, dst + 3 * kN * 32, sh);
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
      }
      __syncwarp();
      if (lane == 0) mbar_arrive(full0 + 8 * slot);
      }
    }
  } else {
    // ---------------- warp 0 lane 0: MMA issue
    if (warp == 0 && lane == 0) {
      for (uint32_t i = 0; i < n_st; ++i) {
        const uint32_t slot = i % kStages;
        mbar_wait(full0 + 8 * slot, (i / kStages) & 1);
        asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
        const uint32_t sb = buf0 + slot * kStageBytes, ta = tmem + kAcol + slot * kAcolsPerStage;
        const uint32_t idesc = half ? kIdescHalf : kIdesc;
#pragma unroll
        for (int s = 0; s < kWords; ++s)
          umma_i8_ta(tmem, ta + s * 8, umma_desc(sb + s * kN * 32), (i | s) ? 1u : 0u, idesc);
        umma_commit(empty0 + 8 * slot);
      }
      umma_commit(done);
    } else if (warp == 1 && lane == 0) {
      // ---------------- TMA: bit stage j = words [word0 + 8 (st0/2 + j), +8) of the A rows and the
      // two 128-row halves of the B rows
      asm volatile("prefetch.tensormap [%0];" ::"l"(&tmap) : "memory");
      const int w0 = (int)(word0 + (uint64_t)st0 * kWords);
      for (uint32_t j = 0; j < n_bst; ++j) {
        const uint32_t bslot = j % kBitStages;
        mbar_wait(bempty0 + 8 * bslot, ((j / kBitStages) & 1) ^ 1);
        const uint32_t bar = bfull0 + 8 * bslot, dst = bits0 + bslot * kBitStageBytes;
        mbar_arrive_expect_tx(bar, half ? (uint32_t)(kM + kBoxRows) * kBitWords * 4 : kBitStageBytes);
        const int c = w0 + (int)(j * kBitWords);
        tma_load_2d(dst, &tmap, c, (int)a0, bar);
        tma_load_2d(dst + kM * 32, &tmap, c, (int)b0, bar);
        if (!half) tma_load_2d(dst + (kM + kBoxRows) * 32, &tmap, c, (int)(b0 + kBoxRows), bar);
      }
    }
    __syncwarp();
    // ---------------- epilogue: warp q reads TMEM lanes 32q..32q+31 (tile rows a), 32 columns at a time
    mbar_wait(done, 0);
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    const uint32_t a = a0 + warp * 32 + lane;
    const uint64_t n = n_rows;
    for (uint32_t c0 = 0; c0 < nN; c0 += 32) {
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

PFN_cuTensorMapEncodeTiled_v12000 get_encode_tc() {
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

uint64_t launch_count_pairs_tc(const uint32_t* rows, uint64_t pitch_words, uint32_t n_rows, uint64_t word_begin,
                               uint64_t word_end, uint32_t* counts, int n_sms, cudaStream_t stream) {
  if (n_rows < 2 || word_end <= word_begin) return 0;
  GPA_REQUIRE(word_begin % kBitWords == 0 && word_end % kBitWords == 0, GPA_ERR_INVALID,
              "count_pairs_tc: word range not a multiple of %d", kBitWords);
  // bit rows as a 2-D tensor {pitch_words, n_rows}; rows >= n_rows read as zeros
  CUtensorMap tmap;
  {
    cuuint64_t dims[2] = {pitch_words, n_rows};
    cuuint64_t strides[1] = {pitch_words * 4};
    cuuint32_t box[2] = {kBitWords, kBoxRows};
    cuuint32_t estr[2] = {1, 1};
    CUresult cr = get_encode_tc()(&tmap, CU_TENSOR_MAP_DATA_TYPE_UINT32, 2, const_cast<uint32_t*>(rows), dims, strides,
                                  box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_32B,
                                  CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    GPA_REQUIRE(cr == CUDA_SUCCESS, GPA_ERR_CUDA, "cuTensorMapEncodeTiled failed (%d)", (int)cr);
  }
  const uint32_t nbi = (n_rows + kM - 1) / kM, nbj = (n_rows + kN - 1) / kN;
  uint64_t live = 0;   // tiles that reach the upper triangle (same enumeration as the kernel)
  for (uint32_t j = 0; j < nbj; ++j) {
    const uint32_t hi = std::min<uint32_t>(n_rows, (j + 1) * kN);
    live += std::min<uint32_t>(nbi, (hi - 1 + kM - 1) / kM);
  }
  const uint64_t n_bst = (word_end - word_begin) / kBitWords;
  GPA_REQUIRE(n_bst < (1ull << 31), GPA_ERR_INVALID, "count_pairs_tc: word range too long");
  // 4 waves of one CTA per SM, at least one CTA per live tile, at most one bit stage per CTA
  uint64_t grid = (uint64_t)n_sms * 4;
  if (grid < live) grid = live;
  if (grid > live * n_bst) grid = live * n_bst;
  GPA_REQUIRE(grid < (1ull << 31), GPA_ERR_INVALID, "count_pairs_tc: grid too large");
  ensure_smem_attr(reinterpret_cast<const void*>(count_pairs_tc_kernel), (int)kSmemBytes);
  {
    count_pairs_tc_kernel<<<(unsigned)grid, kThreads, kSmemBytes, stream>>>(tmap, n_rows, nbi, (uint32_t)live,
                                                                            word_begin, (uint32_t)n_bst, 1u, counts);
    note_launch();
  }
  GPA_CUDA(cudaGetLastError());
  return grid;
}

}  // namespace gpa
