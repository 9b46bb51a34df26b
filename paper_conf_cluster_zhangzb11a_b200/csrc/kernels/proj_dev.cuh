// Device pieces of the projected-list builds (proj.cu): segments, class tables, generation 3's
// word counts.  Internal; included by .cu files only.
#pragma once
#include <cstdint>
#include "../common.h"

namespace gpa {
namespace pj {

constexpr uint32_t kSegJ = 128;          // mask segment: 128 words per lane (a bitset row: 131,072 transactions)
constexpr uint32_t kMemberGroup = 8;     // members sharing one mask preparation in pext_kernel
constexpr uint32_t kG3Group = 16;        // members sharing one chunk's bit ranks in pext3_kernel

struct VecRef {
  const uint32_t* p;
  uint32_t lw;  // words per lane
};

// The mask of a class / the source of a member: a bitset row (generation 3) or one of the
// previous generation's vectors.
struct Src {
  const uint32_t* rows;        // non-null: generation 3
  uint64_t pitch;
  const uint32_t* data;        // previous generation's vectors
  const uint64_t* off;
  const uint32_t* nw;
  __device__ __forceinline__ VecRef vec(uint32_t id) const {
    if (rows) return VecRef{rows + (uint64_t)id * pitch, (uint32_t)(pitch / 32)};
    return VecRef{data + off[id], nw[id] / 32u};
  }
};

__device__ __forceinline__ void seg_range(uint32_t lw, uint32_t s, uint32_t& j0, uint32_t& j1) {
  j0 = min(lw, s * kSegJ);
  j1 = min(lw, j0 + kSegJ);
}

// warp per class c (k >= 4: few segments per class): lane l's output words of every mask segment (the
// lane's set bits rounded up to whole words), their prefix (loc: the lane's word offset of every
// segment), Lw_c = max over lanes of the lane's total, words per member nwc = 32 Lw_c, the class'
// words and its pext items (one per segment with words and group of kMemberGroup members)
__device__ __forceinline__ void seg_pad_warp(uint32_t c, Src src, const uint32_t* __restrict__ par_a,
                                             const uint32_t* __restrict__ bound, uint32_t n_cls, uint32_t cmax,
                                             uint32_t nseg, uint32_t* __restrict__ loc, uint32_t* __restrict__ nwc,
                                             uint64_t* __restrict__ cls_words, uint32_t* __restrict__ items,
                                             uint32_t* __restrict__ max_lw, uint32_t* __restrict__ len,
                                             unsigned long long* __restrict__ in_words) {
  const uint32_t lane = threadIdx.x & 31;
  uint32_t m = 0;
  if (c < n_cls) m = bound[c + 1] - bound[c];
  const uint32_t groups = m >= 2 ? (m + kMemberGroup - 1) / kMemberGroup : 0;
  VecRef mk{nullptr, 0};
  if (groups) mk = src.vec(par_a[bound[c]]);
  uint32_t acc = 0;
  for (uint32_t s = 0; s < nseg; ++s) {
    const uint64_t p = (uint64_t)s * cmax + c;
    uint32_t cnt = 0;
    if (groups) {
      uint32_t a, b;
      seg_range(mk.lw, s, a, b);
      for (uint32_t j = a; j < b; ++j) cnt += __popc(mk.p[32ull * j + lane]);
      if (lane == 0 && b > a) atomicAdd(in_words, 32ull * (b - a) * m);
    }
    const uint32_t w = (cnt + 31) / 32;
    loc[p * 32 + lane] = acc;
    acc += w;
    const bool any = __any_sync(0xffffffffu, w != 0);
    if (lane == 0) items[p] = any ? groups : 0;
  }
  const uint32_t lw = __reduce_max_sync(0xffffffffu, acc);
  len[(uint64_t)c * 32 + lane] = acc;   // lane words written by pext: the rest up to lw is zeroed
  if (lane == 0) {
    nwc[c] = groups ? 32u * lw : 0u;
    cls_words[c] = groups ? (uint64_t)32u * lw * m : 0ull;
    if (groups && lw) atomicMax(max_lw, lw);
  }
}

// generation 3, warp per pair p = s * cmax + c: output words of row a's segment s -- pext3_kernel
// packs the segment's set bits densely across its chunks: ceil(set bits / 32)
__device__ __forceinline__ void seg3_warp(uint32_t p, const uint32_t* __restrict__ rows, uint64_t pitch,
                                          const uint32_t* __restrict__ par_a, const uint32_t* __restrict__ bound,
                                          uint32_t n_cls, uint32_t cmax, uint32_t* __restrict__ w3,
                                          unsigned long long* __restrict__ in_words) {
  const uint32_t lane = threadIdx.x & 31;
  const uint32_t c = p % cmax, s = p / cmax;
  uint32_t words = 0;
  if (c < n_cls) {
    const uint32_t j0 = bound[c], m = bound[c + 1] - j0;
    if (m >= 2) {
      const uint32_t* row = rows + (uint64_t)par_a[j0] * pitch + lane;
      uint32_t a, b;
      seg_range((uint32_t)(pitch / 32), s, a, b);
      uint32_t bits = 0;
      for (uint32_t j = a; j < b; ++j) bits += __popc(row[32ull * j]);
      words = (__reduce_add_sync(0xffffffffu, bits) + 31u) / 32u;
      if (lane == 0 && b > a) atomicAdd(in_words, 32ull * (b - a) * m);
    }
  }
  if (lane == 0) w3[p] = words;
}

// generation 3, thread per class: word offset of every segment in the class' lists, list words (a
// multiple of 32), the class' words, pext3 items (one per segment with words and group of <=
// kG3Group members)
__device__ __forceinline__ void cls3_pad_thread(uint32_t c, const uint32_t* __restrict__ w3,
                                                const uint32_t* __restrict__ bound, uint32_t n_cls, uint32_t cmax,
                                                uint32_t nseg, uint32_t* __restrict__ loc3, uint32_t* __restrict__ nwc,
                                                uint64_t* __restrict__ cls_words, uint32_t* __restrict__ items,
                                                uint32_t* __restrict__ max_lw, uint32_t* __restrict__ len) {
  const uint32_t m = c < n_cls ? bound[c + 1] - bound[c] : 0;
  const uint32_t groups = m >= 2 ? (m + kG3Group - 1) / kG3Group : 0;
  uint32_t acc = 0;
  for (uint32_t s = 0; s < nseg; ++s) {
    const uint64_t p = (uint64_t)s * cmax + c;
    loc3[p] = acc;
    acc += w3[p];
    items[p] = w3[p] ? groups : 0;
  }
  const uint32_t words = groups ? (acc + 31u) & ~31u : 0u;
  len[(uint64_t)c * 32] = acc;   // words written by pext3: the rest up to `words` is zeroed
  nwc[c] = words;
  cls_words[c] = (uint64_t)words * m;
  if (words) atomicMax(max_lw, words / 32u);
}

}  // namespace pj
}  // namespace gpa
