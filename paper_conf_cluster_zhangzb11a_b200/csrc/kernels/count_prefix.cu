// count_prefix -- prefix-staged streaming support counting for any k >= 2 (sm_100a).
//
// Complete intersection (PAPER.md P18@394-1300): supp(P u {e}) = sum_w popc(P[w] & B[e][w])
// with P[w] = AND of the k-1 prefix rows.  Candidates of generation k that share their
// (k-1)-prefix are trie siblings (P13@835-1270, Fig. 4 P18@863); the paper recomputes the full
// k-row AND per candidate.  Here a CTA takes one TASK = (prefix group g, up to 32 siblings)
// and one STRIPE of the transaction (word) axis: each thread ANDs the k-1 prefix rows for its
// U 16-byte slots of the stripe ONCE into registers, then streams the siblings' rows: per
// sibling and 16-byte slot, one LDG.128, 4 LOP3 (AND), 4 POPC and adds.  The per-thread
// partial is reduced across the warp with redux.sync, across warps through shared memory,
// and added to the global count with one atomic per (CTA, sibling) -- integer addition, so
// the result is exact and independent of the order (Q12).
// Grid order is stripe-major (all tasks of stripe 0, then stripe 1, ...) so the rows of the
// stripe being worked on stay resident in the 126 MB L2 and each extension row segment is
// fetched from HBM about once per stripe.  HBM bytes per task-stripe: (k-1+s) x stripe bytes.
#include <cstdint>
#include "../common.h"
#include "../kernels.h"

namespace gpa {
namespace {

constexpr int kPrefixThreads = 256;
constexpr int kPrefixWarps = kPrefixThreads / 32;
constexpr int kU = 2;                                  // 16-byte slots per thread per row
constexpr uint64_t kStripe4 = (uint64_t)kPrefixThreads * kU;   // uint4 per row per stripe (8 KB)

__device__ __forceinline__ uint4 ldg_nc(const uint4* p) { return __ldg(p); }

__global__ void __launch_bounds__(kPrefixThreads) count_prefix_kernel(
    const uint4* __restrict__ rows, uint64_t pitch4, const uint32_t* __restrict__ prefix_rows, uint32_t km1,
    const uint32_t* __restrict__ ext_rows, const PrefixTask* __restrict__ tasks, uint32_t n_tasks,
    uint32_t* __restrict__ counts) {
  __shared__ uint32_t s_pre[GPA_MAX_K];
  __shared__ uint32_t s_ext[kPrefixMaxSiblings];
  __shared__ uint32_t s_red[kPrefixWarps][kPrefixMaxSiblings];
  const uint64_t stripe = blockIdx.x / n_tasks;
  const PrefixTask tk = tasks[blockIdx.x % n_tasks];
  if (threadIdx.x < km1) s_pre[threadIdx.x] = prefix_rows[(uint64_t)tk.group * km1 + threadIdx.x];
  if (threadIdx.x < tk.n) s_ext[threadIdx.x] = ext_rows[tk.first + threadIdx.x];
  __syncthreads();

  const uint64_t base = stripe * kStripe4 + threadIdx.x;
  bool valid[kU];
  uint4 P[kU];
#pragma unroll
  for (int u = 0; u < kU; ++u) {
    valid[u] = base + (uint64_t)u * kPrefixThreads < pitch4;
    P[u] = valid[u] ? ldg_nc(rows + (uint64_t)s_pre[0] * pitch4 + base + u * kPrefixThreads) : make_uint4(0, 0, 0, 0);
  }
  for (uint32_t j = 1; j < km1; ++j) {
    const uint4* r = rows + (uint64_t)s_pre[j] * pitch4 + base;
#pragma unroll
    for (int u = 0; u < kU; ++u) {
      if (valid[u]) {
        const uint4 v = ldg_nc(r + u * kPrefixThreads);
        P[u].x &= v.x; P[u].y &= v.y; P[u].z &= v.z; P[u].w &= v.w;
      }
    }
  }
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
#pragma unroll 2
  for (uint32_t s = 0; s < tk.n; ++s) {
    const uint4* r = rows + (uint64_t)s_ext[s] * pitch4 + base;
    uint32_t acc = 0;
#pragma unroll
    for (int u = 0; u < kU; ++u) {
      if (valid[u]) {
        const uint4 v = ldg_nc(r + u * kPrefixThreads);
        acc += __popc(v.x & P[u].x) + __popc(v.y & P[u].y) + __popc(v.z & P[u].z) + __popc(v.w & P[u].w);
      }
    }
    acc = __reduce_add_sync(0xffffffffu, acc);
    if (lane == 0) s_red[warp][s] = acc;
  }
  __syncthreads();
  if (threadIdx.x < tk.n) {
    uint32_t sum = 0;
#pragma unroll
    for (int w = 0; w < kPrefixWarps; ++w) sum += s_red[w][threadIdx.x];
    if (sum) atomicAdd(&counts[tk.first + threadIdx.x], sum);
  }
}

}  // namespace

uint64_t launch_count_prefix(const uint32_t* rows, uint64_t pitch_words, const uint32_t* prefix_rows, uint32_t km1,
                             const uint32_t* ext_rows, const PrefixTask* tasks, uint32_t n_tasks, uint32_t* counts,
                             cudaStream_t stream) {
  if (n_tasks == 0) return 0;
  const uint64_t pitch4 = pitch_words / 4;
  const uint64_t n_stripes = (pitch4 + kStripe4 - 1) / kStripe4;
  const uint64_t n_blocks = n_stripes * n_tasks;
  GPA_REQUIRE(n_blocks < (1ull << 31), GPA_ERR_INVALID, "count_prefix: grid too large (%llu CTAs)",
              (unsigned long long)n_blocks);
  { count_prefix_kernel<<<(unsigned)n_blocks, kPrefixThreads, 0, stream>>>(
      reinterpret_cast<const uint4*>(rows), pitch4, prefix_rows, km1, ext_rows, tasks, n_tasks, counts); note_launch(); }
  GPA_CUDA(cudaGetLastError());
  return n_blocks;
}

}  // namespace gpa
