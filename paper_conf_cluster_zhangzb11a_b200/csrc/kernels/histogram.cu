// Generation-1 support counting and CSR validation (sm_100a).
//
// "first we generate all 1-item candidates, test their frequencies by scanning the
//  transaction database" (PAPER.md P13@338).  The paper does this on the host; here it is a
// device histogram over the horizontal CSR: one thread per transaction walks its items and
// increments a shared-memory-privatised histogram (flushed with one global atomic per
// non-zero bin per CTA).  The same pass validates the input (offsets monotone, items in
// range) and detects non-canonical transactions (unsorted or duplicated items), for which a
// second, de-duplicating pass counts each item once per transaction (a transaction is a set,
// P3@441).  HBM-bound: reads 8 B/transaction + 4 B/item once.
#include <cstdint>
#include "../common.h"
#include "../kernels.h"

namespace gpa {
namespace {

constexpr int kHistThreads = 256;
constexpr uint32_t kHistSmemMaxItems = 48 * 1024;  // 192 KB of u32 bins

template <bool kSmem>
__global__ void __launch_bounds__(kHistThreads) hist_validate_kernel(const uint64_t* __restrict__ offsets,
                                                                     const uint32_t* __restrict__ items,
                                                                     uint64_t tx_begin, uint64_t n_tx, uint64_t nnz,
                                                                     uint32_t n_items,
                                                                     uint32_t* __restrict__ hist,
                                                                     uint32_t* __restrict__ flags) {
  extern __shared__ uint32_t s_hist[];
  if (kSmem) {
    for (uint32_t i = threadIdx.x; i < n_items; i += blockDim.x) s_hist[i] = 0;
    __syncthreads();
  }
  uint32_t my_flags = 0;
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t t = tx_begin + (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; t < n_tx; t += stride) {
    const uint64_t o0 = __ldg(offsets + t), o1 = __ldg(offsets + t + 1);
    if (o1 < o0 || o1 > nnz) { my_flags |= kFlagBadOffsets; continue; }
    uint32_t prev = 0;
    uint64_t j = o0;
    for (; j + 8 <= o1; j += 8) {  // 8 independent loads in flight
      uint32_t it[8];
#pragma unroll
      for (int u = 0; u < 8; ++u) it[u] = __ldg(items + j + u);
#pragma unroll
      for (int u = 0; u < 8; ++u) {
        if (it[u] >= n_items) { my_flags |= kFlagBadItem; continue; }
        if ((j + u) > o0 && it[u] <= prev) my_flags |= kFlagNonCanonical;
        prev = it[u];
        if (kSmem) atomicAdd(&s_hist[it[u]], 1u);
        else atomicAdd(&hist[it[u]], 1u);
      }
    }
    for (; j < o1; ++j) {
      const uint32_t it = __ldg(items + j);
      if (it >= n_items) { my_flags |= kFlagBadItem; continue; }
      if (j > o0 && it <= prev) my_flags |= kFlagNonCanonical;
      prev = it;
      if (kSmem) atomicAdd(&s_hist[it], 1u);
      else atomicAdd(&hist[it], 1u);
    }
  }
  if (my_flags) atomicOr(flags, my_flags);
  if (kSmem) {
    __syncthreads();
    for (uint32_t i = threadIdx.x; i < n_items; i += blockDim.x)
      if (s_hist[i]) atomicAdd(&hist[i], s_hist[i]);
  }
}

// De-duplicating variant: item j of transaction t counts only if no earlier position of t
// holds the same item (O(len^2) per transaction; only used for non-canonical input).
__global__ void __launch_bounds__(kHistThreads) hist_dedup_kernel(const uint64_t* __restrict__ offsets,
                                                                  const uint32_t* __restrict__ items,
                                                                  uint64_t n_tx, uint64_t nnz, uint32_t n_items,
                                                                  uint32_t* __restrict__ hist) {
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t t = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; t < n_tx; t += stride) {
    const uint64_t o0 = offsets[t], o1 = offsets[t + 1];
    if (o1 < o0 || o1 > nnz) continue;
    for (uint64_t j = o0; j < o1; ++j) {
      const uint32_t it = items[j];
      if (it >= n_items) continue;
      bool first = true;
      for (uint64_t q = o0; q < j && first; ++q) first = items[q] != it;
      if (first) atomicAdd(&hist[it], 1u);
    }
  }
}

int grid_for(uint64_t n_tx, int n_sms) {
  uint64_t want = (n_tx + kHistThreads - 1) / kHistThreads;
  uint64_t cap = (uint64_t)n_sms * 8;
  if (want > cap) want = cap;
  return (int)(want ? want : 1);
}

}  // namespace

void launch_hist_validate_range(const uint64_t* offsets, const uint32_t* items, uint64_t tx_begin, uint64_t tx_end,
                                uint64_t nnz, uint32_t n_items, uint32_t* hist, uint32_t* flags, int n_sms,
                                cudaStream_t stream) {
  if (tx_end <= tx_begin) return;
  const int grid = grid_for(tx_end - tx_begin, n_sms);
  if (n_items <= kHistSmemMaxItems) {
    size_t smem = (size_t)n_items * sizeof(uint32_t);
    if (smem > 48 * 1024)
      GPA_CUDA(cudaFuncSetAttribute(hist_validate_kernel<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    { hist_validate_kernel<true><<<grid, kHistThreads, smem, stream>>>(offsets, items, tx_begin, tx_end, nnz, n_items,
                                                                     hist, flags); note_launch(); }
  } else {
    { hist_validate_kernel<false><<<grid, kHistThreads, 0, stream>>>(offsets, items, tx_begin, tx_end, nnz, n_items,
                                                                   hist, flags); note_launch(); }
  }
  GPA_CUDA(cudaGetLastError());
}

void launch_hist_validate(const uint64_t* offsets, const uint32_t* items, uint64_t n_tx, uint64_t nnz,
                          uint32_t n_items, uint32_t* hist, uint32_t* flags, int n_sms, cudaStream_t stream) {
  launch_hist_validate_range(offsets, items, 0, n_tx, nnz, n_items, hist, flags, n_sms, stream);
}

void launch_hist_dedup(const uint64_t* offsets, const uint32_t* items, uint64_t n_tx, uint64_t nnz, uint32_t n_items,
                       uint32_t* hist, int n_sms, cudaStream_t stream) {
  if (n_tx == 0) return;
  { hist_dedup_kernel<<<grid_for(n_tx, n_sms), kHistThreads, 0, stream>>>(offsets, items, n_tx, nnz, n_items, hist); note_launch(); }
  GPA_CUDA(cudaGetLastError());
}

}  // namespace gpa
