// Single-launch exclusive scans for the level transition (candgen.cu, proj.cu, the plans).
//
// The transition runs a dozen small scans per generation; as CUB calls each is an init kernel, a
// scan kernel and (for the device-side total) a third launch, and on B200 every dependent launch
// costs ~3 us of idle GPU (profiles/r02_microbench_launch_gap.txt).  One kernel per scan here
// (scan_dev.cuh: decoupled look-back, epoch-tagged status words, the total from the last tile).
#include <algorithm>
#include <map>
#include <cstdint>
#include "../common.h"
#include "../kernels.h"
#include "scan_dev.cuh"

namespace gpa {
namespace {

using namespace sd;

template <class T, class TT>
__global__ void __launch_bounds__(kScanThreads, 1) scan_kernel(const T* __restrict__ in, T* __restrict__ out, uint32_t n,
                                                             TT* tot, uint32_t* flags, uint64_t* agg, uint64_t* inc,
                                                             uint32_t epoch) {
  scan_tile<T>(
      n, [&](uint32_t i) { return in[i]; }, [&](uint32_t i, T x, T) { out[i] = x; },
      [&](T t) {
        if (tot) *tot = (TT)t;
      },
      flags, agg, inc, epoch);
}

// (cnt << 32 | cnt != 0) scanned as one u64: off = the running sum of cnt, idx = the running
// number of non-zero cnt; tot2 = {sum, non-zero count}
__global__ void __launch_bounds__(kScanThreads, 1) scan_split_kernel(const uint32_t* __restrict__ cnt,
                                                                   uint32_t* __restrict__ off,
                                                                   uint32_t* __restrict__ idx, uint32_t n,
                                                                   uint32_t* tot2, uint32_t* flags, uint64_t* agg,
                                                                   uint64_t* inc, uint32_t epoch) {
  scan_tile<uint64_t>(
      n,
      [&](uint32_t i) {
        const uint32_t c = cnt[i];
        return ((uint64_t)c << 32) | (uint64_t)(c != 0u);
      },
      [&](uint32_t i, uint64_t x, uint64_t) {
        off[i] = (uint32_t)(x >> 32);
        idx[i] = (uint32_t)x;
      },
      [&](uint64_t t) {
        tot2[0] = (uint32_t)(t >> 32);
        tot2[1] = (uint32_t)t;
      },
      flags, agg, inc, epoch);
}

// two independent exclusive scans in one launch (u32 -> u32 with a u64 total, u64 -> u64): blocks
// [0, t1) run the first, [t1, t1 + t2) the second on status words offset by t1 (a block only waits
// for lower-indexed blocks of its own scan, dispatched first)
__global__ void __launch_bounds__(kScanThreads, 1) dual_scan_kernel(const uint32_t* __restrict__ in1,
                                                                  uint32_t* __restrict__ out1, uint32_t n1,
                                                                  uint64_t* tot1, uint32_t t1,
                                                                  const uint64_t* __restrict__ in2,
                                                                  uint64_t* __restrict__ out2, uint32_t n2,
                                                                  uint64_t* tot2, uint32_t t2, uint32_t* flags,
                                                                  uint64_t* agg, uint64_t* inc, uint32_t epoch) {
  if (blockIdx.x < t1)
    scan_tile<uint32_t>(
        n1, [&](uint32_t i) { return in1[i]; }, [&](uint32_t i, uint32_t x, uint32_t) { out1[i] = x; },
        [&](uint32_t t) { *tot1 = t; }, flags, agg, inc, epoch, 0, t1);
  else
    scan_tile<uint64_t>(
        n2, [&](uint32_t i) { return in2[i]; }, [&](uint32_t i, uint64_t x, uint64_t) { out2[i] = x; },
        [&](uint64_t t) { *tot2 = t; }, flags + t1, agg + t1, inc + t1, epoch, t1, t2);
}

}  // namespace

ScanState& scan_state(int device) {
  thread_local std::map<int, ScanState> m;
  return m[device];
}

uint32_t scan_epoch(ScanState& st, uint32_t tiles, cudaStream_t s) {
  if (st.flags.n < tiles) {   // grow-only (cudaMalloc): fresh flags are zero = no epoch
    const size_t want = std::max<uint32_t>(tiles, 256);
    st.flags.ensure(want);
    st.agg.ensure(st.flags.n);
    st.inc.ensure(st.flags.n);
    GPA_CUDA(cudaMemsetAsync(st.flags.p, 0, st.flags.n * 4, s));
    st.epoch = 0;
  }
  st.epoch = (st.epoch + 1) & ((1u << 30) - 1);
  if (st.epoch == 0) st.epoch = 1;
  return st.epoch;
}
uint32_t scan_tiles(uint32_t n, uint32_t items) {
  const uint32_t tile = kScanThreads * items;
  return (n + tile - 1) / tile;
}

namespace {

template <class T, class TT>
void scan_impl(const T* in, T* out, uint32_t n, TT* tot, ScanState& st, cudaStream_t s) {
  if (n == 0) {
    if (tot) GPA_CUDA(cudaMemsetAsync(tot, 0, sizeof(TT), s));
    return;
  }
  const uint32_t tiles = (n + kScanTile - 1) / kScanTile;
  const uint32_t ep = scan_epoch(st, tiles, s);
  { scan_kernel<T, TT><<<tiles, kScanThreads, 0, s>>>(in, out, n, tot, st.flags.p, st.agg.p, st.inc.p, ep);
    note_launch(); }
  GPA_CUDA(cudaGetLastError());
}

}  // namespace

void scan_excl_u32(const uint32_t* in, uint32_t* out, uint32_t n, uint32_t* tot, ScanState& st, cudaStream_t s) {
  scan_impl<uint32_t, uint32_t>(in, out, n, tot, st, s);
}
void scan_excl_u32(const uint32_t* in, uint32_t* out, uint32_t n, uint64_t* tot, ScanState& st, cudaStream_t s) {
  scan_impl<uint32_t, uint64_t>(in, out, n, tot, st, s);
}
void scan_excl_u64(const uint64_t* in, uint64_t* out, uint32_t n, uint64_t* tot, ScanState& st, cudaStream_t s) {
  scan_impl<uint64_t, uint64_t>(in, out, n, tot, st, s);
}
void scan_excl_split(const uint32_t* cnt, uint32_t* off, uint32_t* idx, uint32_t n, uint32_t* tot2, ScanState& st,
                     cudaStream_t s) {
  if (n == 0) {
    if (tot2) GPA_CUDA(cudaMemsetAsync(tot2, 0, 8, s));
    return;
  }
  const uint32_t tiles = (n + kScanTile - 1) / kScanTile;
  const uint32_t ep = scan_epoch(st, tiles, s);
  { scan_split_kernel<<<tiles, kScanThreads, 0, s>>>(cnt, off, idx, n, tot2, st.flags.p, st.agg.p, st.inc.p, ep);
    note_launch(); }
  GPA_CUDA(cudaGetLastError());
}

void scan_excl_dual(const uint32_t* in1, uint32_t* out1, uint32_t n1, uint64_t* tot1, const uint64_t* in2,
                    uint64_t* out2, uint32_t n2, uint64_t* tot2, ScanState& st, cudaStream_t s) {
  if (n1 == 0 || n2 == 0) {   // (not on the mining path: both are >= 1 there)
    scan_excl_u32(in1, out1, n1, tot1, st, s);
    scan_excl_u64(in2, out2, n2, tot2, st, s);
    return;
  }
  const uint32_t t1 = (n1 + kScanTile - 1) / kScanTile, t2 = (n2 + kScanTile - 1) / kScanTile;
  const uint32_t ep = scan_epoch(st, t1 + t2, s);
  { dual_scan_kernel<<<t1 + t2, kScanThreads, 0, s>>>(in1, out1, n1, tot1, t1, in2, out2, n2, tot2, t2, st.flags.p,
                                                     st.agg.p, st.inc.p, ep); note_launch(); }
  GPA_CUDA(cudaGetLastError());
}

}  // namespace gpa
