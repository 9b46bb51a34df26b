// Device helpers of the level transition shared by candgen.cu (separate kernels) and
// mine_fused.cu (the whole loop in one cooperative launch).  Internal; included by .cu files only.
#pragma once
#include <cstdint>
#include "../common.h"

namespace gpa {
namespace lvl {

__device__ __forceinline__ int lex_cmp(const uint32_t* a, const uint32_t* b, uint32_t w) {
  for (uint32_t i = 0; i < w; ++i)
    if (a[i] != b[i]) return a[i] < b[i] ? -1 : 1;
  return 0;
}

// Open-addressing hash set over the rows of L (slot = row index, 0xffffffff = empty), keyed by
// the polynomial hash H = sum_i (x_i + 1) P^i (mod 2^64) finalised by a mixer.  H is linear in the
// items, so the hash of "x without item d, plus b" is O(1) from per-x prefix / suffix sums.
constexpr uint64_t kHashP = 0x9E3779B97F4A7C15ull | 1ull;
constexpr uint32_t kEmpty = 0xffffffffu;

__device__ __forceinline__ uint64_t hash_mix(uint64_t h) {
  h ^= h >> 33;
  h *= 0xFF51AFD7ED558CCDull;
  h ^= h >> 33;
  return h;
}

__device__ __forceinline__ uint64_t raw_hash(const uint32_t* key, uint32_t w) {
  uint64_t h = 0, p = 1;
  for (uint32_t i = 0; i < w; ++i) {
    h += (uint64_t)(key[i] + 1) * p;
    p *= kHashP;
  }
  return h;
}

// membership of key (w items, raw polynomial hash `raw`) in L
__device__ __forceinline__ bool contains(const uint32_t* __restrict__ L, uint32_t w, const uint32_t* __restrict__ slots,
                                         uint32_t mask, const uint32_t* key, uint64_t raw) {
  uint32_t h = (uint32_t)hash_mix(raw) & mask;
  for (;;) {
    const uint32_t i = slots[h];
    if (i == kEmpty) return false;
    if (lex_cmp(L + (uint64_t)i * w, key, w) == 0) return true;
    h = (h + 1) & mask;
  }
}

// Join + prune of member x of L (n members of w items, lexicographic) with its later run
// siblings, by ONE WARP: lane j tests sibling y = x + 1 + j (+32 ...).  EMIT = false: cnt[x] =
// survivors; EMIT = true: group gidx[x] (prefix = L[x]) and its extensions, in sibling order, at
// cand_off[x] (warp ballot ranks the survivors).  flags / run_ex / bound: run starts, their
// exclusive scan, run boundaries (bound[#runs] = n).
// "px without item d, then b" == L row q?  (no key array: the items are read in place)
__device__ __forceinline__ bool row_is_sub(const uint32_t* __restrict__ row, const uint32_t* __restrict__ px,
                                           uint32_t w, uint32_t d, uint32_t b) {
  for (uint32_t i = 0; i + 1 < w; ++i)
    if (row[i] != px[i < d ? i : i + 1]) return false;
  return row[w - 1] == b;
}

// surv (optional): stage 1 leaves, per member with at most kSurvBits siblings, the bit mask of its
// surviving siblings (bit j: sibling x + 1 + j), kSurvNone otherwise; stage 2 then emits from the
// mask instead of probing the hash set again.
constexpr uint32_t kSurvBits = 63;
constexpr unsigned long long kSurvNone = ~0ull;

template <bool EMIT>
__device__ __forceinline__ void join_warp(uint32_t x, const uint32_t* __restrict__ L, uint32_t w,
                                          const uint32_t* __restrict__ flags, const uint32_t* __restrict__ run_ex,
                                          const uint32_t* __restrict__ bound, const uint32_t* __restrict__ slots,
                                          uint32_t mask, uint32_t* cnt, const uint32_t* __restrict__ cand_off,
                                          const uint32_t* __restrict__ gidx, uint32_t* prefix, uint32_t* ext_off,
                                          uint32_t* ext, uint32_t* gpar, uint32_t* eidx,
                                          unsigned long long* surv = nullptr) {
  const uint32_t lane = threadIdx.x & 31;
  if (EMIT && cnt[x] == 0) return;  // warp-uniform
  const uint32_t* px = L + (uint64_t)x * w;
  if (EMIT && surv) {
    const unsigned long long sm = surv[x];
    if (sm != kSurvNone) {   // the survivors of stage 1: no probes
      const uint32_t base = cand_off[x];
      uint32_t here = 0;
#pragma unroll
      for (uint32_t hf = 0; hf < 2; ++hf) {
        const uint32_t bits = (uint32_t)(sm >> (32 * hf));
        if ((bits >> lane) & 1u) {
          const uint32_t y = x + 1 + 32 * hf + lane;
          const uint32_t at = base + here + __popc(bits & ((1u << lane) - 1u));
          ext[at] = L[(uint64_t)y * w + w - 1];
          eidx[at] = y;
        }
        here += __popc(bits);
      }
      const uint32_t g = gidx[x];
      for (uint32_t i = lane; i < w; i += 32) prefix[(uint64_t)g * w + i] = px[i];
      if (lane == 0) {
        ext_off[g] = base;
        gpar[g] = x;
      }
      return;
    }
  }
  // run index of x = (#run starts <= x) - 1
  const uint32_t r = run_ex[x] + flags[x] - 1;
  const uint32_t end = bound[r + 1];  // bound[n_runs] = n (sentinel end of the last run)
  if (!EMIT && end == x + 1) {
    if (lane == 0) {
      cnt[x] = 0;
      if (surv) surv[x] = 0ull;
    }
    return;
  }
  const bool track = !EMIT && surv && end - x - 1 <= kSurvBits;   // warp-uniform
  unsigned long long smask = 0ull;
  // hash of the subset "px without item d, then b" = A_d + B_d + (b + 1) P^(w-1) with
  // A_d = sum_{i<d} (x_i+1) P^i, B_d = sum_{i>d} (x_i+1) P^(i-1): both walked with d below
  uint64_t B0 = 0, pw = 1;
  for (uint32_t i = 1; i < w; ++i) {
    B0 += (uint64_t)(px[i] + 1) * pw;
    pw *= kHashP;
  }
  const uint64_t p_last = pw;  // P^(w-1)
  uint32_t here = 0;  // survivors so far (warp-uniform)
  const uint32_t np = w - 1;   // prune probes per sibling: the subsets dropping item d < w - 1
  if (np >= 1 && np <= 16) {
    // probes spread over the lanes: lane = (sibling g, item d) for G = 32 / np siblings per round,
    // so a round waits for ONE probe chain instead of np in sequence
    const uint32_t G = 32u / np, d = lane % np, g = lane / np;
    uint64_t hd = 0, pp = 1;   // A_d + B_d: the items of px without d at positions 0 .. w - 2
    for (uint32_t i = 0; i < w; ++i) {
      if (i == d) continue;
      hd += (uint64_t)(px[i] + 1) * pp;
      pp *= kHashP;
    }
    const uint32_t pmask = (1u << np) - 1u;
    for (uint32_t y0 = x + 1; y0 < end; y0 += G) {
      const uint32_t y = y0 + g;
      const bool on = g < G && y < end;
      uint32_t b = 0;
      bool found = true;
      if (on) {
        b = L[(uint64_t)y * w + w - 1];
        uint32_t h = (uint32_t)hash_mix(hd + (uint64_t)(b + 1) * p_last) & mask;
        for (;;) {
          const uint32_t i = slots[h];
          if (i == kEmpty) {
            found = false;
            break;
          }
          if (row_is_sub(L + (uint64_t)i * w, px, w, d, b)) break;
          h = (h + 1) & mask;
        }
      }
      const uint32_t probes = __ballot_sync(0xffffffffu, found);
      // sibling j (lane j < G) survives iff all its np probes hit
      const uint32_t bj = __shfl_sync(0xffffffffu, b, (lane < G ? lane : 0u) * np);
      const bool keep = lane < G && y0 + lane < end && ((probes >> (lane * np)) & pmask) == pmask;
      const uint32_t ballot = __ballot_sync(0xffffffffu, keep);
      if (EMIT && keep) {
        const uint32_t at = cand_off[x] + here + __popc(ballot & ((1u << lane) - 1u));
        ext[at] = bj;
        eidx[at] = y0 + lane;
      }
      if (track) smask |= (unsigned long long)ballot << (y0 - x - 1);   // bits 0 .. G-1 = siblings y0 ..
      here += __popc(ballot);
    }
  } else
  for (uint32_t y0 = x + 1; y0 < end; y0 += 32) {
    const uint32_t y = y0 + lane;
    bool keep = y < end;
    uint32_t b = 0;
    if (keep) {
      b = L[(uint64_t)y * w + w - 1];
      uint64_t A = 0, B = B0, pd = 1;
      const uint64_t hb = (uint64_t)(b + 1) * p_last;
      // subsets dropping item d of the shared prefix (dropping either of the last two items
      // gives the parents x or y, members of L by construction)
      for (uint32_t d = 0; d + 1 < w && keep; ++d) {
        uint32_t h = (uint32_t)hash_mix(A + B + hb) & mask;
        for (;;) {
          const uint32_t i = slots[h];
          if (i == kEmpty) {
            keep = false;
            break;
          }
          if (row_is_sub(L + (uint64_t)i * w, px, w, d, b)) break;
          h = (h + 1) & mask;
        }
        const uint64_t xd = (uint64_t)(px[d] + 1) * pd, xd1 = (uint64_t)(px[d + 1] + 1) * pd;
        A += xd;
        B -= xd1;
        pd *= kHashP;
      }
    }
    const uint32_t ballot = __ballot_sync(0xffffffffu, keep);
    if (EMIT && keep) {
      const uint32_t at = cand_off[x] + here + __popc(ballot & ((1u << lane) - 1u));
      ext[at] = b;
      eidx[at] = y;
    }
    if (track) smask |= (unsigned long long)ballot << (y0 - x - 1);
    here += __popc(ballot);
  }
  if (!EMIT && surv && lane == 0) surv[x] = track ? smask : kSurvNone;
  if (EMIT) {
    const uint32_t g = gidx[x];
    for (uint32_t i = lane; i < w; i += 32) prefix[(uint64_t)g * w + i] = px[i];
    if (lane == 0) {
      ext_off[g] = cand_off[x];
      gpar[g] = x;
    }
  } else if (lane == 0) {
    cnt[x] = here;
  }
}

}  // namespace lvl
}  // namespace gpa
