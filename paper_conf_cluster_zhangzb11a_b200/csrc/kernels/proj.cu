// Projected vertical lists: generation k >= 3 counted on equivalence classes (sm_100a).
//
// The paper contrasts two ways of computing a candidate's vertical list (PAPER.md P13@2288-2486,
// P18@1089): "equivalent class clustering" (Zaki) keeps the vertical lists of generation k-1 and
// intersects two of them, while GPApriori's "complete intersection" re-ANDs k generation-1 rows
// to save memory.  With 180 GB of HBM the first one is affordable once the
// kept lists are stored COMPACTLY: the class of a (k-1)-itemset X = Q u {x} is its (k-2)-prefix
// Q, and the kept list of X is the bit-row of x restricted to the transactions of Q,
//
//     V_X[i] = B[x][t_i],   t_0 < t_1 < ... the transactions containing Q   (|V_X| = supp(Q) bits),
//
// so that every member of a class shares one position list and one bit order, and a candidate
// Q u {a, b} (parents Q u {a}, Q u {b}, P13@1006-1270) has
//
//     supp(Q u {a, b}) = popc(V_{Q u {a}} AND V_{Q u {b}})                 (count_proj_kernel),
//
// the same popcount-of-AND as complete intersection (P18@394), over supp(Q) bits instead of N.
// The next generation's lists follow from this one's: the class of X' = Q u {a, b} is Q u {a},
// whose transactions are the set bits of V_{Q u {a}}; hence V_{X'} = the bits of V_{Q u {b}} at
// the set positions of V_{Q u {a}} (a parallel bit extract).  Generation 3 starts from the static
// bitset itself: the class of a pair {a, b} is {a}, mask = row a, sources = rows b (the "static
// bitset" of P2@270 / P18@755 stays the only input).
//
// B200 design: POSITIONS ONCE PER CLASS, THEN A BALLOT GATHER PER MEMBER.  A class' mask is cut
// into segments of kSegW words (65,536 bits); pos_kernel writes the set-bit positions of each
// (class, segment) once (u16, segment-relative); gather_kernel then gives each warp a (class,
// segment, group of <= 16 members) item: per round of 32 positions, lane l holds position 32r + l,
// loads its word of each member's source list (L1 gather: the 32 positions of a round span a
// few 128-byte lines) and one ballot packs the 32 selected bits into the member's next output
// word.  Work ~ output words (~5 instructions per member and output word), independent of the
// mask's density, with no per-word bit-compress network and no per-member re-ranking of the mask.
// Lists are in natural order (bit i = word i/32, bit i%32), each segment padded to whole words
// and each list to a multiple of 4 words (zero padding is common to the class, so it is never
// selected and never counted).  All integer; counts are exact by construction.
#include <cstdint>
#include <cstdlib>
#include <map>
#include <cub/device/device_scan.cuh>

#include "../common.h"
#include "../kernels.h"

namespace gpa {
namespace {

constexpr int kT = 256;
constexpr uint32_t kSegW = 2048;     // mask segment: 2,048 words = 65,536 bits (u16 positions)
constexpr uint32_t kGroup = 16;      // members per gather item

unsigned grid_for(uint64_t n, int n_sms, int per_sm = 16) {
  uint64_t g = (n + kT - 1) / kT;
  const uint64_t cap = (uint64_t)n_sms * per_sm;
  return (unsigned)(g < 1 ? 1 : (g > cap ? cap : g));
}

// ---------------------------------------------------------------- class structure
// A class = a run of entries with the same par_a (the left parent = the (k-2)-prefix).
__global__ void cls_flag_kernel(const uint32_t* __restrict__ par_a, uint32_t n, uint32_t* __restrict__ flag) {
  for (uint32_t j = blockIdx.x * blockDim.x + threadIdx.x; j < n; j += gridDim.x * blockDim.x)
    flag[j] = j == 0 || par_a[j] != par_a[j - 1];
}

__global__ void cls_bound_kernel(const uint32_t* __restrict__ flag, const uint32_t* __restrict__ ex, uint32_t n,
                                 uint32_t* __restrict__ bound, uint32_t* __restrict__ n_cls) {
  for (uint32_t j = blockIdx.x * blockDim.x + threadIdx.x; j < n; j += gridDim.x * blockDim.x) {
    if (flag[j]) bound[ex[j]] = j;
    if (j == n - 1) {
      const uint32_t C = ex[j] + flag[j];
      bound[C] = n;
      *n_cls = C;
    }
  }
}

// The mask of a class / the source of a member: a bitset row (generation 3) or one of the
// previous generation's lists.  Word offsets are 32-bit (checked by proj_build_begin).
struct Src {
  const uint32_t* base;        // rows (generation 3) or the previous lists' data
  uint64_t pitch;              // generation 3: row pitch (words); 0: lists
  const uint64_t* off;         // lists: word offset of each list
  const uint32_t* nw;          // lists: words of each list
  __device__ __forceinline__ uint32_t offset(uint32_t id) const {
    return pitch ? (uint32_t)(id * pitch) : (uint32_t)off[id];
  }
  __device__ __forceinline__ uint32_t words(uint32_t id) const { return pitch ? (uint32_t)pitch : nw[id]; }
};

__device__ __forceinline__ uint32_t n_segs(uint32_t words) { return (words + kSegW - 1) / kSegW; }

// warp per (segment s, class c) pair p = s * cmax + c: set bits of the class mask in segment s
// -> npos[p] and its output words wseg[p] = ceil(npos / 32); in_words += mask words x members
__global__ void seg_count_kernel(Src src, const uint32_t* __restrict__ par_a, const uint32_t* __restrict__ bound,
                                 const uint32_t* __restrict__ n_cls, uint32_t cmax, uint32_t n_pairs,
                                 uint32_t* __restrict__ npos, uint32_t* __restrict__ wseg,
                                 unsigned long long* __restrict__ in_words) {
  const uint32_t lane = threadIdx.x & 31;
  const uint32_t p = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  if (p >= n_pairs) return;
  const uint32_t c = p % cmax, s = p / cmax;
  uint32_t cnt = 0;
  if (c < *n_cls) {
    const uint32_t j0 = bound[c], m = bound[c + 1] - j0;
    if (m >= 2) {
      const uint32_t mid = par_a[j0];
      const uint32_t W = src.words(mid);
      const uint32_t w0 = s * kSegW, w1 = min(W, w0 + kSegW);
      const uint32_t* mk = src.base + src.offset(mid);
      for (uint32_t w = w0 + 4 * lane; w < w1; w += 128) {   // W is a multiple of 4
        const uint4 v = __ldg(reinterpret_cast<const uint4*>(mk + w));
        cnt += __popc(v.x) + __popc(v.y) + __popc(v.z) + __popc(v.w);
      }
      if (lane == 0 && w1 > w0) atomicAdd(in_words, (unsigned long long)(w1 - w0) * m);
    }
  }
  cnt = __reduce_add_sync(0xffffffffu, cnt);
  if (lane == 0) {
    npos[p] = cnt;
    wseg[p] = (cnt + 31) / 32;
  }
}

// thread per class: the output word offset of every segment of the class (loc), words per member
// nwc = the class total rounded up to 4 words (uint4 loads of count_proj), the class' words, its
// segments and its gather items (one per segment of the mask and group of <= kGroup members)
__global__ void cls_pad_kernel(Src src, const uint32_t* __restrict__ par_a, const uint32_t* __restrict__ wseg,
                               const uint32_t* __restrict__ bound, const uint32_t* __restrict__ n_cls, uint32_t cmax,
                               uint32_t nseg, uint32_t* __restrict__ loc, uint32_t* __restrict__ nwc,
                               uint32_t* __restrict__ cls_nseg, uint64_t* __restrict__ cls_words,
                               uint32_t* __restrict__ items, uint32_t* __restrict__ max_nw) {
  const uint32_t C = *n_cls;
  for (uint32_t c = blockIdx.x * blockDim.x + threadIdx.x; c < cmax; c += gridDim.x * blockDim.x) {
    const uint32_t m = c < C ? bound[c + 1] - bound[c] : 0;
    const uint32_t groups = m >= 2 ? (m + kGroup - 1) / kGroup : 0;
    const uint32_t ns = groups ? n_segs(src.words(par_a[bound[c]])) : 0;
    uint32_t acc = 0;
    for (uint32_t s = 0; s < nseg; ++s) {
      const uint64_t p = (uint64_t)s * cmax + c;
      loc[p] = acc;
      acc += wseg[p];
      items[p] = s < ns ? groups : 0;
    }
    const uint32_t words = groups ? (acc + 3u) & ~3u : 0u;
    nwc[c] = words;
    cls_nseg[c] = ns;
    cls_words[c] = (uint64_t)words * m;
    if (words) atomicMax(max_nw, words);
  }
}

// entry j -> its list (offset, words); entries of single-member classes get none
__global__ void entry_off_kernel(const uint32_t* __restrict__ flag, const uint32_t* __restrict__ ex,
                                 const uint32_t* __restrict__ bound, const uint32_t* __restrict__ nwc,
                                 const uint64_t* __restrict__ cls_base, uint32_t n, uint64_t* __restrict__ off,
                                 uint32_t* __restrict__ nw) {
  for (uint32_t j = blockIdx.x * blockDim.x + threadIdx.x; j < n; j += gridDim.x * blockDim.x) {
    const uint32_t c = ex[j] + flag[j] - 1;
    const uint32_t j0 = bound[c], m = bound[c + 1] - j0;
    if (m < 2) {
      off[j] = 0;
      nw[j] = 0;
    } else {
      nw[j] = nwc[c];
      off[j] = cls_base[c] + (uint64_t)(j - j0) * nwc[c];
    }
  }
}

// warp per pair p with set bits: the segment-relative positions (word << 5 | bit, u16) of the
// class mask's set bits in segment s, in increasing order, at pos + pos_off[p].  128 words per
// step (a uint4 per lane), ranks by a warp scan of the per-lane popcounts.
__global__ void pos_kernel(Src src, const uint32_t* __restrict__ par_a, const uint32_t* __restrict__ bound,
                           uint32_t cmax, uint32_t n_pairs, const uint32_t* __restrict__ npos,
                           const uint64_t* __restrict__ pos_off, uint16_t* __restrict__ pos) {
  const uint32_t lane = threadIdx.x & 31;
  const uint32_t p = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  if (p >= n_pairs || npos[p] == 0) return;
  const uint32_t c = p % cmax, s = p / cmax;
  const uint32_t mid = par_a[bound[c]];
  const uint32_t W = src.words(mid);
  const uint32_t w0 = s * kSegW, w1 = min(W, w0 + kSegW);
  const uint32_t* mk = src.base + src.offset(mid);
  uint16_t* out = pos + pos_off[p];
  uint32_t base = 0;
  for (uint32_t w = w0; w < w1; w += 128) {
    const uint32_t wl = w + 4 * lane;
    const uint4 v = wl < w1 ? __ldg(reinterpret_cast<const uint4*>(mk + wl)) : make_uint4(0, 0, 0, 0);
    const uint32_t t = __popc(v.x) + __popc(v.y) + __popc(v.z) + __popc(v.w);
    uint32_t incl = t;
#pragma unroll
    for (uint32_t d = 1; d < 32; d <<= 1) {
      const uint32_t u = __shfl_up_sync(0xffffffffu, incl, d);
      if (lane >= d) incl += u;
    }
    uint32_t r = base + incl - t;
    const uint32_t rel = (wl - w0) << 5;   // segment-relative bit index of word wl
    const uint32_t x[4] = {v.x, v.y, v.z, v.w};
#pragma unroll
    for (uint32_t i = 0; i < 4; ++i)
      for (uint32_t b = x[i]; b; b &= b - 1u) out[r++] = (uint16_t)(rel + 32u * i + (uint32_t)(__ffs(b) - 1));
    base += __shfl_sync(0xffffffffu, incl, 31);
  }
}

// item -> its pair (items of pair p are item_off[p] .. + items[p])
__global__ void item_pair_kernel(const uint32_t* __restrict__ items, const uint32_t* __restrict__ item_off,
                                 uint32_t n_pairs, uint32_t* __restrict__ item_pair) {
  for (uint32_t p = blockIdx.x * blockDim.x + threadIdx.x; p < n_pairs; p += gridDim.x * blockDim.x)
    for (uint32_t i = 0; i < items[p]; ++i) item_pair[item_off[p] + i] = p;
}

// base + idx words as one IMAD.WIDE.U32 (the scale comes from a kernel parameter so that ptxas
// does not turn the multiply by 4 into LEA + LEA.HI.X on the ALU pipe)
__device__ __forceinline__ const uint32_t* addr_of(const uint32_t* base, uint32_t idx, uint32_t wbytes) {
  const uint32_t* r;
  asm("mad.wide.u32 %0, %1, %2, %3;" : "=l"(r) : "r"(idx), "r"(wbytes), "l"(base));
  return r;
}

// One gather item for G members (G = 2, 4, 8, 16: the unrolled width).  Round r: lane l takes
// position 32 r + l of the segment (0 bits past the last), loads its word of every member's
// source (an L1 gather), and ballot q packs the 32 selected bits of member q into one output word;
// lane (r mod 32) keeps it, and every 32 rounds the lanes store 32 consecutive words per member
// (coalesced).  The positions of the next round are loaded one round ahead.
template <uint32_t G>
__device__ __forceinline__ void gather_item(const uint16_t* __restrict__ P, uint32_t np,
                                            const uint32_t* __restrict__ sb, const uint32_t (&so)[kGroup],
                                            const uint32_t* __restrict__ oo, uint32_t nm,
                                            uint32_t* __restrict__ data, uint32_t wbytes) {
  const uint32_t lane = threadIdx.x & 31;
  uint32_t keep[G];
#pragma unroll
  for (uint32_t q = 0; q < G; ++q) keep[q] = 0;
  const uint32_t rounds = (np + 31) / 32;
  uint32_t vn = lane < np ? (uint32_t)__ldg(P + lane) : 0xffffffffu;
  for (uint32_t r = 0; r < rounds; ++r) {
    const uint32_t v = vn;
    const uint32_t kn = 32u * (r + 1) + lane;
    vn = kn < np ? (uint32_t)__ldg(P + kn) : 0xffffffffu;
    const uint32_t bm = v != 0xffffffffu ? 1u << (v & 31u) : 0u;   // bit select, empty past the end
    const uint32_t* lb = sb + (v != 0xffffffffu ? (v >> 5) : 0u);
    uint32_t x[G];
#pragma unroll
    for (uint32_t q = 0; q < G; ++q) x[q] = __ldg(addr_of(lb, so[q], wbytes));
    const bool mine = lane == (r & 31u);
#pragma unroll
    for (uint32_t q = 0; q < G; ++q) {
      const uint32_t b = __ballot_sync(0xffffffffu, (x[q] & bm) != 0u);
      keep[q] = mine ? b : keep[q];
    }
    if ((r & 31u) == 31u) {
#pragma unroll
      for (uint32_t q = 0; q < G; ++q)
        if (q < nm) data[oo[q] + (r - 31u) + lane] = keep[q];
    }
  }
  if (rounds & 31u) {
    const uint32_t b0 = rounds & ~31u;
    if (lane < (rounds & 31u)) {
#pragma unroll
      for (uint32_t q = 0; q < G; ++q)
        if (q < nm) data[oo[q] + b0 + lane] = keep[q];
    }
  }
}

// Warp per item = (pair p = (segment s, class c), group of <= kGroup members).  Items run
// pair-major = segment-major, so the warps in flight share the same source segments in L2.  The
// item of a class' last segment also zeroes the list tails (words past the class' last segment, up
// to the 4-word padding): every word of every list is written, no memset.
__global__ void __launch_bounds__(kT, 3) gather_kernel(Src src, const uint32_t* __restrict__ par_a,
                                                       const uint32_t* __restrict__ par_b,
                                                       const uint32_t* __restrict__ bound, uint32_t cmax,
                                                       const uint32_t* __restrict__ item_pair,
                                                       const uint32_t* __restrict__ item_off, uint32_t T,
                                                       const uint32_t* __restrict__ npos,
                                                       const uint64_t* __restrict__ pos_off,
                                                       const uint16_t* __restrict__ pos,
                                                       const uint32_t* __restrict__ loc,
                                                       const uint32_t* __restrict__ wseg,
                                                       const uint32_t* __restrict__ nwc,
                                                       const uint32_t* __restrict__ cls_nseg,
                                                       const uint64_t* __restrict__ off,
                                                       uint32_t* __restrict__ data, uint32_t wbytes) {
  __shared__ uint32_t s_oo[kT / 32][kGroup];
  const uint32_t lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const uint32_t it = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  if (it >= T) return;
  (void)par_a;
  const uint32_t p = item_pair[it];
  const uint32_t c = p % cmax, s = p / cmax;
  const uint32_t j0 = bound[c], m = bound[c + 1] - j0;
  const uint32_t g = it - item_off[p];
  const uint32_t first = j0 + g * kGroup;
  const uint32_t nm = min(kGroup, m - g * kGroup);
  uint32_t* oo = s_oo[warp];
  const uint32_t lp = loc[p];
  uint32_t so[kGroup];
#pragma unroll
  for (uint32_t q = 0; q < kGroup; ++q) {
    const uint32_t e = first + (q < nm ? q : 0);  // surplus slots shadow member 0 (not stored)
    so[q] = src.offset(par_b[e]);
    if (lane == q) oo[q] = (uint32_t)off[e] + lp;
  }
  __syncwarp();
  const uint32_t np = npos[p];
  const uint32_t* sb = src.base + (uint64_t)s * kSegW;
  const uint16_t* P = pos + pos_off[p];
  if (nm <= 2)
    gather_item<2>(P, np, sb, so, oo, nm, data, wbytes);
  else if (nm <= 4)
    gather_item<4>(P, np, sb, so, oo, nm, data, wbytes);
  else if (nm <= 8)
    gather_item<8>(P, np, sb, so, oo, nm, data, wbytes);
  else
    gather_item<16>(P, np, sb, so, oo, nm, data, wbytes);
  if (s + 1 == cls_nseg[c]) {   // zero the tail of the members' lists
    const uint32_t w_end = lp + wseg[p], W = nwc[c];
    for (uint32_t q = 0; q < nm; ++q) {
      const uint32_t base = oo[q] - lp;
      for (uint32_t w = w_end + lane; w < W; w += 32) data[base + w] = 0u;
    }
  }
}

// ---------------------------------------------------------------- counting
// WARP = false: CTA per group g (left parent x = gpar[g]), its warps striding over 256-word chunks
// of the class lists, one atomic per (warp, sibling) -- long lists (generation 3); WARP = true:
// one warp per group walking the whole list, plain stores -- short lists (deep generations, where
// a CTA per group would leave most of its warps idle).  Siblings in batches of 32 (lane j
// accumulates sibling j); two siblings share one packed redux.sync (per-chunk warp sums
// <= 32 x 8 x 32 < 2^16).  Lists hold a multiple of 4 words, zero-padded.
template <bool WARP>
__global__ void __launch_bounds__(kT) count_proj_kernel(const uint32_t* __restrict__ data,
                                                        const uint64_t* __restrict__ off,
                                                        const uint32_t* __restrict__ nw,
                                                        const uint32_t* __restrict__ gpar,
                                                        const uint32_t* __restrict__ ext_off,
                                                        const uint32_t* __restrict__ eidx,
                                                        uint32_t* __restrict__ counts, uint32_t G) {
  const uint32_t lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const uint32_t g = WARP ? blockIdx.x * (kT / 32) + warp : blockIdx.x;
  if (WARP && g >= G) return;
  constexpr uint32_t w_step = WARP ? 256u : (kT / 32) * 256u;
  const uint32_t x = gpar[g];
  const uint32_t n = nw[x];
  const uint32_t* X = data + off[x];
  const uint32_t e0 = ext_off[g], e1 = ext_off[g + 1];
  for (uint32_t b0 = e0; b0 < e1; b0 += 32) {
    const uint32_t nb = min(32u, e1 - b0);
    const uint64_t my_off = lane < nb ? off[eidx[b0 + lane]] : 0;
    uint32_t acc = 0;
    for (uint32_t w = WARP ? 0u : warp * 256u; w < n; w += w_step) {
      const uint32_t w0 = w + lane * 4, w1 = w + 128 + lane * 4;
      const bool h0 = w0 < n, h1 = w1 < n;
      const uint4 x0 = h0 ? *reinterpret_cast<const uint4*>(X + w0) : make_uint4(0, 0, 0, 0);
      const uint4 x1 = h1 ? *reinterpret_cast<const uint4*>(X + w1) : make_uint4(0, 0, 0, 0);
      for (uint32_t i = 0; i < nb; i += 2) {
        uint32_t c = 0;
#pragma unroll
        for (uint32_t q = 0; q < 2; ++q) {
          if (i + q < nb) {
            const uint64_t yo = __shfl_sync(0xffffffffu, my_off, i + q);
            const uint32_t* Y = data + yo;
            const uint4 y0 = h0 ? *reinterpret_cast<const uint4*>(Y + w0) : make_uint4(0, 0, 0, 0);
            const uint4 y1 = h1 ? *reinterpret_cast<const uint4*>(Y + w1) : make_uint4(0, 0, 0, 0);
            const uint32_t v = __popc(x0.x & y0.x) + __popc(x0.y & y0.y) + __popc(x0.z & y0.z) +
                               __popc(x0.w & y0.w) + __popc(x1.x & y1.x) + __popc(x1.y & y1.y) +
                               __popc(x1.z & y1.z) + __popc(x1.w & y1.w);
            c |= v << (16 * q);
          }
        }
        c = __reduce_add_sync(0xffffffffu, c);
        if (lane == i) acc += c & 0xffffu;
        if (lane == i + 1) acc += c >> 16;
      }
    }
    if (WARP) {
      if (lane < nb) counts[b0 + lane] = acc;
    } else if (lane < nb && acc) {
      atomicAdd(&counts[b0 + lane], acc);
    }
  }
}

template <class T>
void scan_excl(const T* in, T* out, uint32_t n, PBuf<uint8_t>& tmpbuf, cudaStream_t s) {
  size_t bytes = 0;
  GPA_CUDA(cub::DeviceScan::ExclusiveSum(nullptr, bytes, in, out, n, s));
  void* tmp = tmpbuf.ensure(bytes);
  GPA_CUDA(cub::DeviceScan::ExclusiveSum(tmp, bytes, in, out, n, s));
  note_launch(2);
}

// totals: tot[0] = gather items, tot[1] = list words, tot[2] = positions
__global__ void proj_totals_kernel(const uint32_t* __restrict__ items, const uint32_t* __restrict__ item_off,
                                   uint32_t n_pairs, const uint64_t* __restrict__ cw, const uint64_t* __restrict__ cb,
                                   uint32_t cmax, const uint32_t* __restrict__ npos,
                                   const uint64_t* __restrict__ pos_off, uint64_t* __restrict__ tot) {
  if (threadIdx.x == 0 && blockIdx.x == 0) {
    tot[0] = (uint64_t)item_off[n_pairs - 1] + items[n_pairs - 1];
    tot[1] = cb[cmax - 1] + cw[cmax - 1];
    tot[2] = pos_off[n_pairs - 1] + npos[n_pairs - 1];
  }
}

// u32 -> u64 widening (the positions' offsets are scanned in 64 bits)
__global__ void widen_kernel(const uint32_t* __restrict__ in, uint64_t* __restrict__ out, uint32_t n) {
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) out[i] = in[i];
}

// per-thread, per-device persistent workspace (grow-only): the class tables of proj_build and the
// two generations of lists
struct ProjWork {
  PBuf<uint32_t> flag, ex, bound, small, npos, wseg, loc, items, item_off, item_pair, nwc, cls_nseg;
  PBuf<uint64_t> cls_words, cls_base, tot, npos64, pos_off;
  PBuf<uint16_t> pos;
  PBuf<uint8_t> tmp;   // CUB temporary storage of its own: proj_build_begin may run beside the join's scans
  DeviceProj lists[2];
};
ProjWork& work_for(int device) {
  thread_local std::map<int, ProjWork> w;
  return w[device];
}

Src make_src(const ProjPending& pp) {
  Src src{};
  if (!pp.prev) {
    src.base = pp.rows;
    src.pitch = pp.pitch;
  } else {
    src.base = pp.prev->data.p;
    src.off = pp.prev->off.p;
    src.nw = pp.prev->nw.p;
  }
  return src;
}

}  // namespace

DeviceProj* proj_lists(int device) { return work_for(device).lists; }

bool proj_build_begin(uint32_t n, const uint32_t* par_a, const uint32_t* par_b, const DeviceProj* prev,
                      const uint32_t* rows, uint64_t pitch_words, uint32_t n_rows, DeviceScratch& scratch, int n_sms,
                      cudaStream_t s, ProjPending& pp) {
  (void)scratch;
  pp = ProjPending();
  pp.n = n;
  pp.par_a = par_a;
  pp.par_b = par_b;
  pp.prev = prev;
  pp.rows = rows;
  pp.pitch = pitch_words;
  if (n == 0) return true;
  const Src src = make_src(pp);
  const uint32_t cmax = prev ? n : std::min(n, n_rows);
  const uint64_t w_max = prev ? prev->max_nw : pitch_words;
  const uint32_t nseg = (uint32_t)std::max<uint64_t>(1, (w_max + kSegW - 1) / kSegW);
  // sources are addressed with 32-bit word offsets, the tables with 31-bit thread indices: beyond
  // that the caller uses complete intersection
  if (!prev && (uint64_t)n_rows * pitch_words >= (1ull << 32)) return false;
  if (prev && prev->words >= (1ull << 32)) return false;
  const uint64_t n_pairs64 = (uint64_t)cmax * nseg;
  if (n_pairs64 * 32 >= (1ull << 31)) return false;
  const uint32_t n_pairs = (uint32_t)n_pairs64;
  pp.cmax = cmax;
  pp.nseg = nseg;
  pp.n_pairs = n_pairs;
  GPA_CUDA(cudaGetDevice(&pp.device));
  ProjWork& W = work_for(pp.device);
  W.flag.ensure(n);
  W.ex.ensure(n);
  W.bound.ensure(n + 1);
  W.small.ensure(4);
  GPA_CUDA(cudaMemsetAsync(W.small.p, 0, 16, s));
  { cls_flag_kernel<<<grid_for(n, n_sms), kT, 0, s>>>(par_a, n, W.flag.p); note_launch(); }
  scan_excl<uint32_t>(W.flag.p, W.ex.p, n, W.tmp, s);
  { cls_bound_kernel<<<grid_for(n, n_sms), kT, 0, s>>>(W.flag.p, W.ex.p, n, W.bound.p, W.small.p); note_launch(); }
  W.npos.ensure(n_pairs);
  W.wseg.ensure(n_pairs);
  W.loc.ensure(n_pairs);
  W.items.ensure(n_pairs);
  W.item_off.ensure(n_pairs);
  W.npos64.ensure(n_pairs);
  W.pos_off.ensure(n_pairs);
  W.nwc.ensure(cmax);
  W.cls_nseg.ensure(cmax);
  W.cls_words.ensure(cmax);
  W.cls_base.ensure(cmax);
  W.tot.ensure(3);
  const unsigned wpb = kT / 32;
  { seg_count_kernel<<<(n_pairs + wpb - 1) / wpb, kT, 0, s>>>(src, par_a, W.bound.p, W.small.p, cmax, n_pairs,
        W.npos.p, W.wseg.p, reinterpret_cast<unsigned long long*>(W.small.p + 2)); note_launch(); }
  { cls_pad_kernel<<<grid_for(cmax, n_sms), kT, 0, s>>>(src, par_a, W.wseg.p, W.bound.p, W.small.p, cmax, nseg,
        W.loc.p, W.nwc.p, W.cls_nseg.p, W.cls_words.p, W.items.p, W.small.p + 1); note_launch(); }
  { widen_kernel<<<grid_for(n_pairs, n_sms), kT, 0, s>>>(W.npos.p, W.npos64.p, n_pairs); note_launch(); }
  scan_excl<uint32_t>(W.items.p, W.item_off.p, n_pairs, W.tmp, s);
  scan_excl<uint64_t>(W.cls_words.p, W.cls_base.p, cmax, W.tmp, s);
  scan_excl<uint64_t>(W.npos64.p, W.pos_off.p, n_pairs, W.tmp, s);
  { proj_totals_kernel<<<1, 32, 0, s>>>(W.items.p, W.item_off.p, n_pairs, W.cls_words.p, W.cls_base.p, cmax,
                                        W.npos.p, W.pos_off.p, W.tot.p); note_launch(); }
  GPA_CUDA(cudaGetLastError());
  pp.d_tot = W.tot.p;
  pp.d_small = W.small.p;
  return true;
}

bool proj_build_finish(const ProjPending& pp, const uint64_t T[3], const uint32_t sm[4], DeviceProj& out, int n_sms,
                       cudaStream_t s, cudaEvent_t ev_build) {
  const uint32_t n = pp.n;
  out.n = n;
  out.words = 0;
  out.in_words = 0;
  if (n == 0) {
    if (ev_build) GPA_CUDA(cudaEventRecord(ev_build, s));
    return true;
  }
  if (T[0] >= (1ull << 31) || T[1] >= (1ull << 32)) return false;
  // GPA_PROJ_MAX_MB caps the lists of one generation (tests exercise the mid-run fallback to
  // complete intersection with it; default: no cap beyond device memory)
  if (const char* cap = getenv("GPA_PROJ_MAX_MB"))
    if (T[1] * 4 > (uint64_t)atof(cap) * 1e6) return false;
  ProjWork& W = work_for(pp.device);
  try {
    out.data.ensure(T[1]);
    W.pos.ensure(T[2]);
  } catch (const Error& e) {
    if (e.status != GPA_ERR_OOM) throw;
    return false;  // caller falls back to complete intersection
  }
  const Src src = make_src(pp);
  out.off.ensure(n);
  out.nw.ensure(n);
  out.words = T[1];
  out.max_nw = sm[1];
  out.max_lw = (sm[1] + 31) / 32;
  out.in_words = (uint64_t)sm[2] | ((uint64_t)sm[3] << 32);
  const unsigned wpb = kT / 32;
  { entry_off_kernel<<<grid_for(n, n_sms), kT, 0, s>>>(W.flag.p, W.ex.p, W.bound.p, W.nwc.p, W.cls_base.p, n,
                                                      out.off.p, out.nw.p); note_launch(); }
  if (ev_build) GPA_CUDA(cudaEventRecord(ev_build, s));  // start of the list build proper
  if (T[0]) {
    W.item_pair.ensure(T[0]);
    { item_pair_kernel<<<grid_for(pp.n_pairs, n_sms), kT, 0, s>>>(W.items.p, W.item_off.p, pp.n_pairs,
                                                                 W.item_pair.p); note_launch(); }
    if (T[2])
      { pos_kernel<<<(pp.n_pairs + wpb - 1) / wpb, kT, 0, s>>>(src, pp.par_a, W.bound.p, pp.cmax, pp.n_pairs,
                                                               W.npos.p, W.pos_off.p, W.pos.p); note_launch(); }
    const uint64_t blocks = (T[0] + wpb - 1) / wpb;
    { gather_kernel<<<(unsigned)blocks, kT, 0, s>>>(src, pp.par_a, pp.par_b, W.bound.p, pp.cmax, W.item_pair.p,
                                                    W.item_off.p, (uint32_t)T[0], W.npos.p, W.pos_off.p, W.pos.p,
                                                    W.loc.p, W.wseg.p, W.nwc.p, W.cls_nseg.p, out.off.p, out.data.p,
                                                    4u); note_launch(); }
  }
  GPA_CUDA(cudaGetLastError());
  return true;
}

void launch_count_proj(const DeviceProj& P, const uint32_t* gpar, const uint32_t* ext_off, const uint32_t* eidx,
                       uint32_t G, uint32_t* counts, cudaStream_t s) {
  if (G == 0) return;
  if ((uint64_t)P.max_nw <= 8192)
    { count_proj_kernel<true><<<(G + kT / 32 - 1) / (kT / 32), kT, 0, s>>>(P.data.p, P.off.p, P.nw.p, gpar, ext_off,
                                                                          eidx, counts, G); note_launch(); }
  else
    { count_proj_kernel<false><<<G, kT, 0, s>>>(P.data.p, P.off.p, P.nw.p, gpar, ext_off, eidx, counts, G);
      note_launch(); }
  GPA_CUDA(cudaGetLastError());
}

}  // namespace gpa
