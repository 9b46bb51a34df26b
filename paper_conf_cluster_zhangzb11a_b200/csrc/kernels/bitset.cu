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
//   transactions (kPer consecutive items per thread, kPer item loads in flight), sets bits with
//   shared-memory atomicOr (duplicates are harmless: OR is idempotent, so non-canonical input
//   needs no special case), then writes every row's 64-byte segment with coalesced stores.  Every word of the output is written (padding
//   transactions contribute no bits, so padding is zero).
#include <algorithm>
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
constexpr uint32_t kPer = 8;             // items per thread and round of the sweep
constexpr uint32_t kSmemRowMap = 1024;   // item -> row map in shared memory up to this many items (3 CTAs / SM)

__global__ void __launch_bounds__(kBuildThreads) bitset_build_kernel(const uint64_t* __restrict__ offsets,
                                                                     const uint32_t* __restrict__ items,
                                                                     uint64_t n_tx, uint64_t nnz,
                                                                     const int32_t* __restrict__ row_of_item,
                                                                     uint32_t n_items, uint32_t n_rows, uint32_t row_block,
                                                                     uint64_t chunk0,
                                                                     uint64_t pitch_words, uint32_t* __restrict__ rows) {
  extern __shared__ uint32_t tile[];
  __shared__ uint32_t soff[kChunkTx + 1];        // the chunk's offsets, relative to its first item
  __shared__ int32_t srow[kSmemRowMap];          // row_of_item (n_items <= kSmemRowMap)
  const uint64_t chunk = chunk0 + blockIdx.x;
  const uint32_t rb0 = blockIdx.y * row_block;
  const uint32_t nr = min(row_block, n_rows - rb0);
  const bool smap = n_items <= kSmemRowMap;
  for (uint32_t i = threadIdx.x; i < nr * kTileStride; i += blockDim.x) tile[i] = 0;
  if (smap)
    for (uint32_t i = threadIdx.x; i < n_items; i += blockDim.x) srow[i] = __ldg(row_of_item + i);
  // item range of the chunk, clamped so that an invalid CSR (rejected by the validation pass)
  // never reads past the items or out of the tile
  const uint64_t t0 = chunk * kChunkTx;
  const uint64_t te = t0 < n_tx ? t0 : n_tx;
  const uint64_t A = min(__ldg(offsets + te), nnz);
  for (uint32_t i = threadIdx.x; i <= kChunkTx; i += blockDim.x) {
    const uint64_t t = t0 + i < n_tx ? t0 + i : n_tx;
    const uint64_t o = min(max(__ldg(offsets + t), A), nnz);
    soff[i] = (uint32_t)(o - A < 0xffffffffull ? o - A : 0xffffffffull);
  }
  __syncthreads();
  // coalesced sweep over the chunk's items: thread k takes items kPer*k .. kPer*k + kPer-1 (+ kPer x 256
  // per round; kPer loads in flight per thread); the transaction of its first item by binary search in
  // soff, then a forward walk
  const uint32_t n_it = soff[kChunkTx];
  for (uint32_t q = threadIdx.x * kPer; q < n_it; q += blockDim.x * kPer) {
    uint32_t it[kPer];
#pragma unroll
    for (int u = 0; u < (int)kPer; ++u) it[u] = q + u < n_it ? __ldg(items + A + q + u) : 0xffffffffu;
    uint32_t lo = 0, hi = kChunkTx;  // tx = last with soff[tx] <= q
    while (lo + 1 < hi) {
      const uint32_t mid = (lo + hi) >> 1;
      if (soff[mid] <= q) lo = mid; else hi = mid;
    }
    uint32_t tx = lo;
#pragma unroll
    for (int u = 0; u < (int)kPer; ++u) {
      const uint32_t j = q + u;
      if (j >= n_it) break;
      while (tx + 1 < kChunkTx && soff[tx + 1] <= j) ++tx;
      const uint32_t x = it[u];
      const int32_t r = x < n_items ? (smap ? srow[x] : __ldg(row_of_item + x)) : -1;
      const uint32_t rr = (uint32_t)r - rb0;   // r < 0 wraps to a huge value: skipped
      if (r >= 0 && rr < nr) atomicOr(&tile[rr * kTileStride + (tx >> 5)], 1u << (tx & 31));
    }
  }
  __syncthreads();
  uint32_t* out = rows + (uint64_t)rb0 * pitch_words + chunk * kChunkWords;
  for (uint32_t i = threadIdx.x; i < nr * kChunkWords; i += blockDim.x) {
    const uint32_t r = i / kChunkWords, w = i % kChunkWords;
    out[(uint64_t)r * pitch_words + w] = tile[r * kTileStride + w];
  }
}

// ---------------------------------------------------------------- one pass: histogram + bitset
// Generation 1 AND the static bitset from ONE read of the CSR (the database is read once, as
// the paper copies it once, P18@755): CTA = one 512-transaction chunk, a shared-memory tile of
// ALL n_items rows (identity row map; n_items <= kScanMaxItems), the chunk's items streamed into
// shared memory by cp.async.bulk (double-buffered 16 KB pieces: bytes in flight without
// registers), bits set with shared atomicOr, then every row's 64-byte segment written out and its
// popcount added to hist[item] -- the generation-1 count with set semantics (a duplicate item
// sets the same bit; P3@441), so non-canonical input needs no de-duplication pass.  Validation:
// offsets monotone and <= nnz, items < n_items (flags).
constexpr uint32_t kScanMaxItems = 1024;
constexpr uint32_t kPiece = 4096;          // items per bulk-copy piece (16 KB)
constexpr int kScanThreads = 512;          // 2 CTAs (112 KB of shared memory each) = 32 warps per SM
constexpr uint32_t kScanStride = 20;       // tile row stride (words): 16-byte aligned rows for LDS/STS.128

__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return (uint32_t)__cvta_generic_to_shared(p);
}

__global__ void __launch_bounds__(kScanThreads) scan_build_kernel(const uint64_t* __restrict__ offsets,
                                                                  const uint32_t* __restrict__ items,
                                                                  uint64_t n_tx, uint64_t nnz, uint32_t n_items,
                                                                  uint64_t chunk0, uint64_t pitch_words,
                                                                  uint32_t* __restrict__ rows,
                                                                  uint32_t* __restrict__ hist,
                                                                  uint32_t* __restrict__ flags) {
  extern __shared__ __align__(16) uint32_t dyn[];
  uint32_t* buf = dyn;                                   // 2 x (kPiece + 4) items (16-byte aligned pieces)
  uint32_t* tile = dyn + 2 * (kPiece + 4);               // n_items x kScanStride words
  __shared__ uint32_t soff[kChunkTx + 1];
  __shared__ __align__(8) uint64_t bar[2];
  __shared__ uint32_t s_flags;
  const uint32_t lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const uint64_t chunk = chunk0 + blockIdx.x;
  for (uint32_t i = threadIdx.x; i < n_items * (kScanStride / 4); i += blockDim.x)
    reinterpret_cast<uint4*>(tile)[i] = make_uint4(0, 0, 0, 0);
  if (threadIdx.x == 0) {
    s_flags = 0;
    asm volatile("mbarrier.init.shared.b64 [%0], 1;" ::"r"(smem_u32(&bar[0])));
    asm volatile("mbarrier.init.shared.b64 [%0], 1;" ::"r"(smem_u32(&bar[1])));
    asm volatile("fence.mbarrier_init.release.cluster;");
  }
  const uint64_t t0 = chunk * kChunkTx;
  const uint64_t te = t0 < n_tx ? t0 : n_tx;
  const uint64_t A = min(__ldg(offsets + te), nnz);
  uint32_t my_flags = 0;
  for (uint32_t i = threadIdx.x; i <= kChunkTx; i += blockDim.x) {
    const uint64_t t = t0 + i < n_tx ? t0 + i : n_tx;
    const uint64_t o_raw = __ldg(offsets + t);
    if (o_raw > nnz) my_flags |= kFlagBadOffsets;
    if (i > 0 && t0 + i <= n_tx && o_raw < __ldg(offsets + t - 1)) my_flags |= kFlagBadOffsets;
    const uint64_t o = min(max(o_raw, A), nnz);
    soff[i] = (uint32_t)(o - A < 0xffffffffull ? o - A : 0xffffffffull);
  }
  __syncthreads();
  const uint32_t n_it = soff[kChunkTx];
  // pieces: items [A + p kPiece, ...) copied from the 16-byte aligned index at or below (the
  // items pointer is 16-byte aligned, checked by the launcher), never past the last whole 16-byte
  // group of the array: the last <= 3 items of the array are stored into the buffer by the issuer
  const uint64_t cend = nnz & ~3ull;
  const uint32_t n_pieces = (n_it + kPiece - 1) / kPiece;
  auto issue = [&](uint32_t p) {
    const uint64_t first = A + (uint64_t)p * kPiece;
    const uint64_t last = A + min(n_it, (p + 1) * kPiece);       // exclusive
    const uint64_t a0 = first & ~3ull, a1r = (last + 3) & ~3ull;
    const uint64_t a1 = a1r < cend ? a1r : cend;
    if (a1 <= a0) {   // nothing copyable (the array's tail only): complete the phase without a copy
      for (uint64_t x = first; x < last; ++x) buf[(p & 1) * (kPiece + 4) + (uint32_t)(x - (first & ~3ull))] = __ldg(items + x);
      asm volatile("mbarrier.arrive.shared.b64 _, [%0];" ::"r"(smem_u32(&bar[p & 1])) : "memory");
      return;
    }
    // the array's last items past the last whole 16-byte group (never bulk-copied) are stored by
    // this thread before its arrive, so that every item of the piece is read from shared memory
    for (uint64_t x = max(first, cend); x < last; ++x) buf[(p & 1) * (kPiece + 4) + (uint32_t)(x - a0)] = __ldg(items + x);
    const uint32_t bytes = (uint32_t)((a1 - a0) * 4);
    const uint32_t b = smem_u32(&bar[p & 1]);
    asm volatile("mbarrier.arrive.expect_tx.shared.b64 _, [%0], %1;" ::"r"(b), "r"(bytes) : "memory");
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                 ::"r"(smem_u32(buf + (p & 1) * (kPiece + 4))), "l"(items + a0), "r"(bytes), "r"(b) : "memory");
  };
  if (threadIdx.x == 0 && n_pieces > 0) {
    issue(0);
    if (n_pieces > 1) issue(1);
  }
  const uint32_t head0 = (uint32_t)(A & 3ull);   // every piece starts at a multiple of kPiece: same head
  for (uint32_t p = 0; p < n_pieces; ++p) {
    const uint32_t b = smem_u32(&bar[p & 1]);
    const uint32_t parity = (p >> 1) & 1;
    asm volatile("{ .reg .pred P; WAIT_%=: mbarrier.try_wait.parity.shared.b64 P, [%0], %1; @!P bra WAIT_%=; }"
                 ::"r"(b), "r"(parity) : "memory");
    const uint32_t q0 = p * kPiece, q1 = min(n_it, q0 + kPiece);
    const uint4* pb = reinterpret_cast<const uint4*>(buf + (p & 1) * (kPiece + 4));   // 16-byte groups
    // warp step = 32 aligned 16-byte groups of the buffer (128 items, one conflict-free LDS.128 per
    // lane); group g holds items q0 - head0 + 4g .. + 3 (chunk-relative, 32-bit).  Each lane finds
    // the transaction of its first item by a binary search over soff, the next ones by comparing
    // with the next transaction's start (kept in a register)
    const uint32_t n_groups = (head0 + (q1 - q0) + 3) / 4;
    for (uint32_t g = warp * 32 + lane; g - lane < n_groups; g += kScanThreads) {
      if (g >= n_groups) continue;
      const uint4 v = pb[g];
      const uint32_t xs[4] = {v.x, v.y, v.z, v.w};
      const int32_t jr0 = (int32_t)(q0 + 4 * g) - (int32_t)head0;   // chunk-relative index of xs[0]
      const uint32_t ja = (uint32_t)max(jr0, (int32_t)q0);
      uint32_t lo = 0, hi = kChunkTx;   // last tx with soff[tx] <= ja
#pragma unroll
      for (int it = 0; it < 9; ++it) {
        const uint32_t mid = (lo + hi) >> 1;
        const bool le = soff[mid] <= ja;
        lo = le ? mid : lo;
        hi = le ? hi : mid;
      }
      uint32_t tx = lo, nxt = soff[lo + 1];   // soff[512] = n_it > any item stops the walk
      uint32_t* trow = tile + (tx >> 5);
      uint32_t bit = 1u << (tx & 31);
#pragma unroll
      for (int i = 0; i < 4; ++i) {
        const int32_t jr = jr0 + i;
        if (jr < (int32_t)q0 || jr >= (int32_t)q1) continue;
        const uint32_t j = (uint32_t)jr;
        if (j >= nxt) {
          do nxt = soff[++tx + 1]; while (j >= nxt);
          trow = tile + (tx >> 5);
          bit = 1u << (tx & 31);
        }
        const uint32_t x = xs[i];
        if (x < n_items) atomicOr(trow + x * kScanStride, bit);
        else my_flags |= kFlagBadItem;
      }
    }
    __syncthreads();   // every thread is done with buffer p & 1
    if (threadIdx.x == 0 && p + 2 < n_pieces) issue(p + 2);
  }
  // out: a quad of lanes per row (4 x 16 bytes = the row's 64-byte segment, STG.128), the row's
  // popcount into the histogram
  uint32_t* out = rows + chunk * kChunkWords;
  const uint32_t quad = lane & 3;
  for (uint32_t r = threadIdx.x >> 2; r < ((n_items + 7) & ~7u); r += kScanThreads / 4) {
    uint4 v = make_uint4(0, 0, 0, 0);
    if (r < n_items) {
      v = *reinterpret_cast<const uint4*>(tile + r * kScanStride + 4 * quad);
      *reinterpret_cast<uint4*>(out + (uint64_t)r * pitch_words + 4 * quad) = v;
    }
    uint32_t c = __popc(v.x) + __popc(v.y) + __popc(v.z) + __popc(v.w);
    c += __shfl_xor_sync(0xffffffffu, c, 1);
    c += __shfl_xor_sync(0xffffffffu, c, 2);
    if (quad == 0 && r < n_items && c) atomicAdd(&hist[r], c);
  }
  if (my_flags) atomicOr(&s_flags, my_flags);
  __syncthreads();
  if (threadIdx.x == 0 && s_flags) atomicOr(flags, s_flags);
}

// In-place compaction of a full bitset (row = item id) to the rows of the selected items
// (sel ascending, sel[r] >= r): row r <- row sel[r] for r >= r0.  Each thread owns a column of
// 16-byte words and walks the rows in increasing r; a row is only read at an iteration <= the one
// that overwrites it (sel[r] >= r), so per-address program order makes it race-free.
__global__ void compact_rows_kernel(uint4* __restrict__ rows, const uint32_t* __restrict__ sel, uint32_t r0,
                                    uint32_t n_sel, uint64_t pitch4) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < pitch4; i += (uint64_t)gridDim.x * blockDim.x)
    for (uint32_t r = r0; r < n_sel; ++r) rows[(uint64_t)r * pitch4 + i] = rows[(uint64_t)sel[r] * pitch4 + i];
}

}  // namespace

bool scan_build_supported(uint32_t n_items, const void* items) {
  return n_items >= 1 && n_items <= kScanMaxItems && ((uintptr_t)items & 15) == 0;
}

void launch_scan_build(const uint64_t* offsets, const uint32_t* items, uint64_t n_tx, uint64_t nnz, uint32_t n_items,
                       uint64_t pitch_words, uint32_t* rows, uint32_t* hist, uint32_t* flags, cudaStream_t stream) {
  GPA_REQUIRE(scan_build_supported(n_items, items), GPA_ERR_INVALID, "scan_build: n_items %u or items unaligned",
              n_items);
  const uint64_t n_chunks = pitch_words / kChunkWords;   // the padding chunks write zeros
  GPA_REQUIRE(n_chunks < (1ull << 31), GPA_ERR_INVALID, "scan_build: too many transactions");
  const size_t smem = (2 * (kPiece + 4) + (size_t)n_items * kScanStride) * sizeof(uint32_t);
  ensure_smem_attr(reinterpret_cast<const void*>(scan_build_kernel), (int)smem);
  { scan_build_kernel<<<(unsigned)n_chunks, kScanThreads, smem, stream>>>(offsets, items, n_tx, nnz, n_items, 0,
                                                                         pitch_words, rows, hist, flags);
    note_launch(); }
  GPA_CUDA(cudaGetLastError());
}

void launch_compact_rows(uint32_t* rows, const uint32_t* sel, uint32_t r0, uint32_t n_sel, uint64_t pitch_words,
                         int n_sms, cudaStream_t stream) {
  if (r0 >= n_sel) return;
  const uint64_t pitch4 = pitch_words / 4;
  const uint64_t want = (pitch4 + 255) / 256;
  const unsigned grid = (unsigned)std::min<uint64_t>(want, (uint64_t)n_sms * 8);
  { compact_rows_kernel<<<grid, 256, 0, stream>>>(reinterpret_cast<uint4*>(rows), sel, r0, n_sel, pitch4);
    note_launch(); }
  GPA_CUDA(cudaGetLastError());
}

void launch_bitset_build(const uint64_t* offsets, const uint32_t* items, uint64_t n_tx, uint64_t nnz,
                         const int32_t* row_of_item,
                         uint32_t n_items, uint32_t n_rows, uint64_t pitch_words, uint32_t* rows, uint64_t tx_begin,
                         uint64_t tx_end, cudaStream_t stream) {
  if (n_rows == 0 || tx_end <= tx_begin) return;
  GPA_REQUIRE(tx_begin % kChunkTx == 0, GPA_ERR_INVALID, "bitset: range start not aligned");
  const uint64_t c0 = tx_begin / kChunkTx;
  // the range that ends at n_tx also writes the (zero) padding chunks up to the pitch
  const uint64_t c1 = tx_end >= n_tx ? pitch_words / kChunkWords
                                     : std::min<uint64_t>((tx_end + kChunkTx - 1) / kChunkTx, pitch_words / kChunkWords);
  const uint32_t rb = n_rows < kRowBlock ? n_rows : kRowBlock;
  const uint32_t n_rb = (n_rows + rb - 1) / rb;
  const size_t smem = (size_t)rb * kTileStride * sizeof(uint32_t);
  GPA_CUDA(cudaFuncSetAttribute(bitset_build_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  GPA_REQUIRE(c1 - c0 < (1ull << 31), GPA_ERR_INVALID, "bitset: too many transactions");
  dim3 grid((unsigned)(c1 - c0), n_rb);
  { bitset_build_kernel<<<grid, kBuildThreads, smem, stream>>>(offsets, items, n_tx, nnz, row_of_item, n_items, n_rows, rb, c0,
                                                             pitch_words, rows); note_launch(); }
  GPA_CUDA(cudaGetLastError());
}

namespace {
__global__ void pairs_subset_kernel(const uint32_t* __restrict__ all, uint32_t n_all, const uint32_t* __restrict__ sel,
                                    uint32_t n_sub, uint32_t* __restrict__ sub) {
  // one warp per a, lanes over b
  const uint32_t warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5, lane = threadIdx.x & 31;
  const uint32_t n_warps = (gridDim.x * blockDim.x) >> 5;
  for (uint32_t a = warp; a + 1 < n_sub; a += n_warps) {
    const uint64_t src0 = pair_index(sel[a], sel[a] + 1, n_all) - (sel[a] + 1);
    const uint64_t dst0 = pair_index(a, a + 1, n_sub) - (a + 1);
    for (uint32_t b = a + 1 + lane; b < n_sub; b += 32) sub[dst0 + b] = all[src0 + sel[b]];
  }
}
__global__ void gather_rows_kernel(const uint4* __restrict__ all, const uint32_t* __restrict__ sel, uint32_t n_sub,
                                   uint64_t pitch4, uint4* __restrict__ sub) {
  for (uint32_t r = blockIdx.y; r < n_sub; r += gridDim.y) {
    const uint4* src = all + (uint64_t)sel[r] * pitch4;
    uint4* dst = sub + (uint64_t)r * pitch4;
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < pitch4; i += (uint64_t)gridDim.x * blockDim.x)
      dst[i] = __ldg(src + i);
  }
}
}  // namespace

void launch_pairs_subset(const uint32_t* counts_all, uint32_t n_all, const uint32_t* sel, uint32_t n_sub,
                         uint32_t* counts_sub, int n_sms, cudaStream_t stream) {
  if (n_sub < 2) return;
  { pairs_subset_kernel<<<n_sms * 4, 256, 0, stream>>>(counts_all, n_all, sel, n_sub, counts_sub); note_launch(); }
  GPA_CUDA(cudaGetLastError());
}

void launch_gather_rows(const uint32_t* rows_all, const uint32_t* sel, uint32_t n_sub, uint64_t pitch_words,
                        uint32_t* rows_sub, int n_sms, cudaStream_t stream) {
  if (n_sub == 0) return;
  const uint64_t pitch4 = pitch_words / 4;
  unsigned gx = (unsigned)std::min<uint64_t>((pitch4 + 255) / 256, 64);
  dim3 grid(gx, std::min<uint32_t>(n_sub, 65535));
  { gather_rows_kernel<<<grid, 256, 0, stream>>>(reinterpret_cast<const uint4*>(rows_all), sel, n_sub, pitch4,
                                               reinterpret_cast<uint4*>(rows_sub)); note_launch(); }
  GPA_CUDA(cudaGetLastError());
}

}  // namespace gpa
