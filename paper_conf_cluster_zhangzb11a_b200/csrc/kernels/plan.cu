// Device-side work planning for the counting kernels (sm_100a), so that a generation's
// candidates never leave the GPU between candidate generation and counting.
//
//  * trie kernel plan (count_trie.cu): blocks of <= kTrieMaxCand lexicographically consecutive
//    candidates touching <= rmax distinct rows.  Windows of 256 candidates are tested in parallel
//    (one CTA per window: a shared-memory bitmap over the rows, popcount); windows over the limit
//    are halved and retested (a few passes), which yields the same kind of blocks as the host
//    greedy plan (runtime/candgen.cpp plan_trie).  Then one CTA per block writes the block's row
//    list (bitmap order = ascending row), every candidate's block-local row bytes and its shared
//    prefix length with its predecessor (0 at every warp-chunk start).
//  * prefix kernel tasks (count_prefix.cu): (group, first sibling, <= 32 siblings).
#include <cstdint>

#include "../common.h"
#include "../kernels.h"

namespace gpa {
namespace {

constexpr int kThreads = 256;
constexpr uint32_t kMaxBitmapWords = kPlanMaxRows / 32;

__global__ void cand_group_kernel(const uint32_t* __restrict__ ext_off, uint32_t G, uint32_t* cand_group) {
  for (uint32_t g = blockIdx.x * blockDim.x + threadIdx.x; g < G; g += gridDim.x * blockDim.x)
    for (uint32_t m = ext_off[g]; m < ext_off[g + 1]; ++m) cand_group[m] = g;
}

__device__ __forceinline__ uint32_t cand_item(const uint32_t* __restrict__ prefix, const uint32_t* __restrict__ ext,
                                              const uint32_t* __restrict__ cand_group, uint32_t km1, uint32_t m,
                                              uint32_t d) {
  return d < km1 ? prefix[(uint64_t)cand_group[m] * km1 + d] : ext[m];
}

// Distinct rows of each window [start, start + len): R[w].
__global__ void window_rows_kernel(const uint32_t* __restrict__ prefix, const uint32_t* __restrict__ ext,
                                   const uint32_t* __restrict__ cand_group, uint32_t k, uint32_t n_rows,
                                   const uint2* __restrict__ windows, uint32_t* R) {
  __shared__ uint32_t bm[kMaxBitmapWords];
  __shared__ uint32_t s_cnt;
  const uint32_t nw = (n_rows + 31) / 32;
  const uint2 win = windows[blockIdx.x];
  for (uint32_t i = threadIdx.x; i < nw; i += blockDim.x) bm[i] = 0;
  if (threadIdx.x == 0) s_cnt = 0;
  __syncthreads();
  for (uint32_t i = threadIdx.x; i < win.y * k; i += blockDim.x) {
    const uint32_t r = cand_item(prefix, ext, cand_group, k - 1, win.x + i / k, i % k);
    atomicOr(&bm[r >> 5], 1u << (r & 31));
  }
  __syncthreads();
  uint32_t c = 0;
  for (uint32_t i = threadIdx.x; i < nw; i += blockDim.x) c += __popc(bm[i]);
  c = __reduce_add_sync(0xffffffffu, c);
  if ((threadIdx.x & 31) == 0) atomicAdd(&s_cnt, c);
  __syncthreads();
  if (threadIdx.x == 0) R[blockIdx.x] = s_cnt;
}

// One CTA per final block: row list, local row bytes and lcp of its candidates.
__global__ void build_blocks_kernel(const uint32_t* __restrict__ prefix, const uint32_t* __restrict__ ext,
                                    const uint32_t* __restrict__ cand_group, uint32_t k, uint32_t n_rows,
                                    TrieBlock* __restrict__ blocks, uint32_t* trows, uint4* lrows,
                                    uint8_t* lcp) {
  __shared__ uint32_t bm[kMaxBitmapWords];
  __shared__ uint32_t base[kMaxBitmapWords];
  const uint32_t nw = (n_rows + 31) / 32;
  const TrieBlock blk = blocks[blockIdx.x];
  for (uint32_t i = threadIdx.x; i < nw; i += blockDim.x) bm[i] = 0;
  __syncthreads();
  for (uint32_t i = threadIdx.x; i < blk.n_cand * k; i += blockDim.x) {
    const uint32_t r = cand_item(prefix, ext, cand_group, k - 1, blk.cand_begin + i / k, i % k);
    atomicOr(&bm[r >> 5], 1u << (r & 31));
  }
  __syncthreads();
  if (threadIdx.x == 0) {  // exclusive prefix popcount over the bitmap words (<= 2,048 words)
    uint32_t acc = 0;
    for (uint32_t i = 0; i < nw; ++i) {
      base[i] = acc;
      acc += __popc(bm[i]);
    }
    blocks[blockIdx.x].n_rows = acc;  // exact count (the host may have planned with an upper bound)
  }
  __syncthreads();
  for (uint32_t i = threadIdx.x; i < nw; i += blockDim.x) {
    uint32_t w = bm[i], l = base[i];
    while (w) {
      const uint32_t b = __ffs(w) - 1;
      w &= w - 1;
      trows[blk.row_begin + l++] = i * 32 + b;
    }
  }
  const uint32_t chunk = (blk.n_cand + 7) / 8;  // the kernel's even split over 8 warps
  for (uint32_t c = threadIdx.x; c < blk.n_cand; c += blockDim.x) {
    const uint32_t m = blk.cand_begin + c;
    uint8_t bytes[16] = {0};
    uint32_t l = 0;
    bool same = c % chunk != 0;
    for (uint32_t d = 0; d < k; ++d) {
      const uint32_t r = cand_item(prefix, ext, cand_group, k - 1, m, d);
      bytes[d] = (uint8_t)(base[r >> 5] + __popc(bm[r >> 5] & ((1u << (r & 31)) - 1u)));
      if (same && d + 1 < k && cand_item(prefix, ext, cand_group, k - 1, m - 1, d) == r) ++l;
      else same = false;
    }
    uint32_t w[4];
    for (int q = 0; q < 4; ++q)
      w[q] = bytes[4 * q] | (bytes[4 * q + 1] << 8) | (bytes[4 * q + 2] << 16) | ((uint32_t)bytes[4 * q + 3] << 24);
    lrows[m] = make_uint4(w[0], w[1], w[2], w[3]);
    lcp[m] = (uint8_t)l;
  }
}

// prefix-kernel tasks: group g has ceil(size / 32) tasks starting at task_off[g]
__global__ void task_count_kernel(const uint32_t* __restrict__ ext_off, uint32_t G, uint32_t* n_tasks) {
  for (uint32_t g = blockIdx.x * blockDim.x + threadIdx.x; g < G; g += gridDim.x * blockDim.x)
    n_tasks[g] = (ext_off[g + 1] - ext_off[g] + kPrefixMaxSiblings - 1) / kPrefixMaxSiblings;
}
__global__ void task_write_kernel(const uint32_t* __restrict__ ext_off, uint32_t G, const uint32_t* __restrict__ task_off,
                                  PrefixTask* tasks) {
  for (uint32_t g = blockIdx.x * blockDim.x + threadIdx.x; g < G; g += gridDim.x * blockDim.x) {
    uint32_t t = task_off[g];
    for (uint32_t j = ext_off[g]; j < ext_off[g + 1]; j += kPrefixMaxSiblings)
      tasks[t++] = PrefixTask{g, j, min(kPrefixMaxSiblings, ext_off[g + 1] - j), 0};
  }
}

unsigned grid_for(uint64_t n, int n_sms) {
  uint64_t g = (n + kThreads - 1) / kThreads;
  const uint64_t cap = (uint64_t)n_sms * 16;
  return (unsigned)(g < 1 ? 1 : (g > cap ? cap : g));
}

}  // namespace

void launch_cand_group(const uint32_t* ext_off, uint32_t G, uint32_t* cand_group, int n_sms, cudaStream_t s) {
  if (G == 0) return;
  cand_group_kernel<<<grid_for(G, n_sms), kThreads, 0, s>>>(ext_off, G, cand_group);
  GPA_CUDA(cudaGetLastError());
}

void launch_window_rows(const uint32_t* prefix, const uint32_t* ext, const uint32_t* cand_group, uint32_t k,
                        uint32_t n_rows, const uint2* windows, uint32_t n_windows, uint32_t* R, cudaStream_t s) {
  if (n_windows == 0) return;
  window_rows_kernel<<<n_windows, kThreads, 0, s>>>(prefix, ext, cand_group, k, n_rows, windows, R);
  GPA_CUDA(cudaGetLastError());
}

void launch_build_blocks(const uint32_t* prefix, const uint32_t* ext, const uint32_t* cand_group, uint32_t k,
                         uint32_t n_rows, TrieBlock* blocks, uint32_t n_blocks, uint32_t* trows, uint4* lrows,
                         uint8_t* lcp, cudaStream_t s) {
  if (n_blocks == 0) return;
  build_blocks_kernel<<<n_blocks, kThreads, 0, s>>>(prefix, ext, cand_group, k, n_rows, blocks, trows, lrows, lcp);
  GPA_CUDA(cudaGetLastError());
}

void launch_prefix_tasks(const uint32_t* ext_off, uint32_t G, uint32_t* n_tasks, const uint32_t* task_off,
                         PrefixTask* tasks, int n_sms, cudaStream_t s, bool write) {
  if (G == 0) return;
  if (!write) task_count_kernel<<<grid_for(G, n_sms), kThreads, 0, s>>>(ext_off, G, n_tasks);
  else task_write_kernel<<<grid_for(G, n_sms), kThreads, 0, s>>>(ext_off, G, task_off, tasks);
  GPA_CUDA(cudaGetLastError());
}

}  // namespace gpa
