// The single-launch exclusive scan's device part (scan.cu), for kernels that fuse their own input
// transform / output side effects into the scan (candgen.cu, proj.cu).  Internal.
//
// CTA = tile of 256 x ITEMS values (8 by default; fewer for input transforms with dependent loads,
// so that more CTAs are in flight), block scan in registers + shuffles, the tile's
// prefix by decoupled look-back over the earlier tiles' published aggregate / inclusive values.
// The status words carry the scan's epoch (ScanState, one per stream), so no init pass clears them
// between scans.  Tiles are blockIdx order: a tile only waits for lower-indexed tiles, which the
// hardware dispatches first.  Launch: scan_tiles(n, ITEMS) CTAs of kScanThreads with scan_epoch()'s
// epoch.
#pragma once
#include <cstdint>
#include "../common.h"

namespace gpa {
namespace sd {

constexpr int kScanThreads = 256;
constexpr int kScanItems = 8;
constexpr uint32_t kScanTile = kScanThreads * kScanItems;

__device__ __forceinline__ void st_release(uint32_t* p, uint32_t v) {
  asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ uint32_t ld_acquire(const uint32_t* p) {
  uint32_t v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}

template <class T>
__device__ __forceinline__ T warp_incl(T v, uint32_t lane) {
#pragma unroll
  for (uint32_t d = 1; d < 32; d <<= 1) {
    const T t = __shfl_up_sync(0xffffffffu, v, d);
    if (lane >= d) v += t;
  }
  return v;
}

// in(i): value of element i < n; out(i, exclusive prefix, value); tot(total) by the last tile.
// Several scans in one launch: blocks [tile0, tile0 + n_tiles) run this one (its own status words:
// flags / agg / inc already offset by the caller); n_tiles = 0: the whole grid.
template <class T, int ITEMS = kScanItems, class In, class Out, class Tot>
__device__ __forceinline__ void scan_tile(uint32_t n, In in, Out out, Tot tot, uint32_t* __restrict__ flags,
                                          uint64_t* __restrict__ agg, uint64_t* __restrict__ inc, uint32_t epoch,
                                          uint32_t tile0 = 0, uint32_t n_tiles = 0) {
  __shared__ T s_warp[kScanThreads / 32];
  __shared__ T s_prefix;
  const uint32_t tile = blockIdx.x - tile0, lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const uint32_t last_tile = (n_tiles ? n_tiles : gridDim.x) - 1;
  const uint32_t base = tile * (kScanThreads * ITEMS) + threadIdx.x * ITEMS;
  T v[ITEMS];
  T sum = 0;
#pragma unroll
  for (int j = 0; j < ITEMS; ++j) {
    v[j] = base + j < n ? in(base + j) : T(0);
    sum += v[j];
  }
  const T wi = warp_incl(sum, lane);
  if (lane == 31) s_warp[warp] = wi;
  __syncthreads();
  if (warp == 0) {
    T x = lane < kScanThreads / 32 ? s_warp[lane] : T(0);
    const T xi = warp_incl(x, lane);
    if (lane < kScanThreads / 32) s_warp[lane] = xi - x;   // exclusive warp offsets
    const T aggregate = __shfl_sync(0xffffffffu, xi, kScanThreads / 32 - 1);
    T prefix = 0;
    if (tile == 0) {
      if (lane == 0) {
        inc[0] = (uint64_t)aggregate;
        st_release(&flags[0], (epoch << 2) | 2u);
      }
    } else {
      if (lane == 0) {
        agg[tile] = (uint64_t)aggregate;
        st_release(&flags[tile], (epoch << 2) | 1u);
      }
      // look back 32 tiles at a time until a published inclusive prefix
      int pred = (int)tile - 1;
      for (;;) {
        const int idx = pred - (int)lane;
        uint32_t st = 2;
        T val = 0;
        if (idx >= 0) {
          uint32_t f;
          do {
            f = ld_acquire(&flags[idx]);
          } while ((f >> 2) != epoch || (f & 3u) == 0u);
          st = f & 3u;
          val = (T)(st == 2u ? __ldcg(inc + idx) : __ldcg(agg + idx));
        }
        const uint32_t b = __ballot_sync(0xffffffffu, st == 2u);
        const uint32_t first = b ? (uint32_t)__ffs(b) - 1u : 32u;   // lanes before tile 0 count as inclusive 0
        T c = lane <= first ? val : T(0);   // the nearest inclusive tile and the aggregates before it
#pragma unroll
        for (uint32_t d = 16; d; d >>= 1) c += __shfl_xor_sync(0xffffffffu, c, d);
        prefix += c;
        if (first < 32) break;
        pred -= 32;
      }
      if (lane == 0) {
        inc[tile] = (uint64_t)(prefix + aggregate);
        st_release(&flags[tile], (epoch << 2) | 2u);
      }
    }
    if (lane == 0) {
      s_prefix = prefix;
      if (tile == last_tile) tot(prefix + aggregate);
    }
  }
  __syncthreads();
  T run = s_prefix + s_warp[warp] + (wi - sum);
#pragma unroll
  for (int j = 0; j < ITEMS; ++j) {
    if (base + j < n) out(base + j, run, v[j]);
    run += v[j];
  }
}

}  // namespace sd
}  // namespace gpa
