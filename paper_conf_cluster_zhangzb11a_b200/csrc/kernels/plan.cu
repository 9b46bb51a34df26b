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

// Greedy block partition of each window of <= 256 consecutive candidates (one CTA per window; the
// walk is sequential like the host plan_trie, rows tracked in a shared-memory bitmap): a block is
// closed when the next candidate would bring it over rmax distinct rows.  Writes up to 256 block
// records per window (x = first candidate, y = count, z = distinct rows) and their number.
__global__ void window_greedy_kernel(const uint32_t* __restrict__ prefix, const uint32_t* __restrict__ ext,
                                     const uint32_t* __restrict__ cand_group, uint32_t k, uint32_t n_rows, uint32_t M,
                                     uint32_t window, uint32_t rmax, uint3* recs, uint32_t* n_recs) {
  __shared__ uint32_t bm[kMaxBitmapWords];
  __shared__ uint32_t items[kTrieMaxCand * kTrieMaxK];   // the window's candidates, staged cooperatively
  const uint32_t nw = (n_rows + 31) / 32;
  const uint32_t c0 = blockIdx.x * window, c1 = min(c0 + window, M);
  for (uint32_t i = threadIdx.x; i < nw; i += blockDim.x) bm[i] = 0;
  for (uint32_t i = threadIdx.x; i < (c1 - c0) * k; i += blockDim.x)
    items[i] = cand_item(prefix, ext, cand_group, k - 1, c0 + i / k, i % k);
  __syncthreads();
  if (threadIdx.x >= 32) return;
  // warp 0 walks the candidates; lane d < k tests / sets the bit of item d (items of one candidate
  // are distinct, so the k bit updates never collide)
  const uint32_t lane = threadIdx.x;
  uint32_t n = 0, start = c0, rows = 0;
  for (uint32_t m = c0; m < c1; ++m) {
    const uint32_t r = lane < k ? items[(m - c0) * k + lane] : 0;
    const bool fresh_bit = lane < k && !((bm[r >> 5] >> (r & 31)) & 1u);
    uint32_t fresh = __popc(__ballot_sync(0xffffffffu, fresh_bit));
    if (rows + fresh > rmax) {  // close [start, m)
      if (lane == 0) recs[(uint64_t)blockIdx.x * window + n] = make_uint3(start, m - start, rows);
      ++n;
      __syncwarp();
      for (uint32_t i = lane; i < nw; i += 32) bm[i] = 0;
      __syncwarp();
      start = m;
      rows = 0;
      fresh = k;
    }
    if (lane < k) atomicOr(&bm[r >> 5], 1u << (r & 31));
    __syncwarp();
    rows += fresh;
  }
  if (lane == 0 && c1 > start) recs[(uint64_t)blockIdx.x * window + n] = make_uint3(start, c1 - start, rows);
  if (c1 > start) ++n;
  if (lane != 0) return;
  n_recs[blockIdx.x] = n;
}

// Compact the per-window records into the block table (row_begin filled later); rows[b] = the
// block's distinct rows; stats[0] = max rows over blocks (atomicMax)
__global__ void compact_blocks_kernel(const uint3* __restrict__ recs, const uint32_t* __restrict__ n_recs,
                                      const uint32_t* __restrict__ off, uint32_t n_win, uint32_t window,
                                      TrieBlock* blocks, uint32_t* rows, uint32_t* stats) {
  for (uint32_t w = blockIdx.x; w < n_win; w += gridDim.x)
    for (uint32_t i = threadIdx.x; i < n_recs[w]; i += blockDim.x) {
      const uint3 r = recs[(uint64_t)w * window + i];
      blocks[off[w] + i] = TrieBlock{r.x, r.y, 0, r.z};
      rows[off[w] + i] = r.z;
      atomicMax(&stats[0], r.z);
    }
}
__global__ void row_begin_kernel(const uint32_t* __restrict__ row_off, uint32_t n_blocks, TrieBlock* blocks) {
  for (uint32_t b = blockIdx.x * blockDim.x + threadIdx.x; b < n_blocks; b += gridDim.x * blockDim.x)
    blocks[b].row_begin = row_off[b];
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
  { cand_group_kernel<<<grid_for(G, n_sms), kThreads, 0, s>>>(ext_off, G, cand_group); note_launch(); }
  GPA_CUDA(cudaGetLastError());
}

void launch_window_rows(const uint32_t* prefix, const uint32_t* ext, const uint32_t* cand_group, uint32_t k,
                        uint32_t n_rows, const uint2* windows, uint32_t n_windows, uint32_t* R, cudaStream_t s) {
  if (n_windows == 0) return;
  { window_rows_kernel<<<n_windows, kThreads, 0, s>>>(prefix, ext, cand_group, k, n_rows, windows, R); note_launch(); }
  GPA_CUDA(cudaGetLastError());
}

void launch_window_greedy(const uint32_t* prefix, const uint32_t* ext, const uint32_t* cand_group, uint32_t k,
                          uint32_t n_rows, uint32_t M, uint32_t window, uint32_t rmax, uint3* recs, uint32_t* n_recs,
                          cudaStream_t s) {
  if (M == 0) return;
  const uint32_t n_win = (M + window - 1) / window;
  { window_greedy_kernel<<<n_win, 64, 0, s>>>(prefix, ext, cand_group, k, n_rows, M, window, rmax, recs, n_recs); note_launch(); }
  GPA_CUDA(cudaGetLastError());
}

void launch_compact_blocks(const uint3* recs, const uint32_t* n_recs, const uint32_t* off, uint32_t n_win,
                           uint32_t window, TrieBlock* blocks, uint32_t* rows, uint32_t* stats, cudaStream_t s) {
  if (n_win == 0) return;
  { compact_blocks_kernel<<<n_win < 4096 ? n_win : 4096, 64, 0, s>>>(recs, n_recs, off, n_win, window, blocks, rows, stats); note_launch(); }
  GPA_CUDA(cudaGetLastError());
}

void launch_row_begin(const uint32_t* row_off, uint32_t n_blocks, TrieBlock* blocks, int n_sms, cudaStream_t s) {
  if (n_blocks == 0) return;
  { row_begin_kernel<<<grid_for(n_blocks, n_sms), kThreads, 0, s>>>(row_off, n_blocks, blocks); note_launch(); }
  GPA_CUDA(cudaGetLastError());
}

void launch_build_blocks(const uint32_t* prefix, const uint32_t* ext, const uint32_t* cand_group, uint32_t k,
                         uint32_t n_rows, TrieBlock* blocks, uint32_t n_blocks, uint32_t* trows, uint4* lrows,
                         uint8_t* lcp, cudaStream_t s) {
  if (n_blocks == 0) return;
  { build_blocks_kernel<<<n_blocks, kThreads, 0, s>>>(prefix, ext, cand_group, k, n_rows, blocks, trows, lrows, lcp); note_launch(); }
  GPA_CUDA(cudaGetLastError());
}

void launch_prefix_tasks(const uint32_t* ext_off, uint32_t G, uint32_t* n_tasks, const uint32_t* task_off,
                         PrefixTask* tasks, int n_sms, cudaStream_t s, bool write) {
  if (G == 0) return;
  if (!write) { task_count_kernel<<<grid_for(G, n_sms), kThreads, 0, s>>>(ext_off, G, n_tasks); note_launch(); }
  else { task_write_kernel<<<grid_for(G, n_sms), kThreads, 0, s>>>(ext_off, G, task_off, tasks); note_launch(); }
  GPA_CUDA(cudaGetLastError());
}

}  // namespace gpa
