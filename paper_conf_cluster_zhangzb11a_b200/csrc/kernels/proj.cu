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
// the set positions of V_{Q u {a}}: a parallel bit extract, pext(V_{Q u {b}}, V_{Q u {a}}),
// word by word (pext_kernel; Hacker's Delight "compress", the mask-dependent half computed once
// per mask word and shared by a warp's group of up to 8 members of the class).  Generation 3 starts from the static
// bitset itself: the class of a pair {a, b} is {a}, mask = row a, sources = rows b (the "static
// bitset" of P2@270 / P18@755 stays the only input).
//
// Layout: LANE-INTERLEAVED.  A vector is 32 bit streams ("lanes") of Lw words each, word j of
// lane l at index 32 j + l; a bitset row is such a vector with Lw = pitch / 32.  Lane l of a new
// vector is the pext of lane l of its source by lane l of its mask, so a warp's lane l only ever
// touches lane l: every load is a coalesced 128-byte row, no cross-lane bit placement.  The
// members of a class share one mask, hence one per-lane bit count and one layout: Lw_c = max
// over lanes of the lane's words (each lane's tail zero-padded), members contiguous.  A bitset
// mask is cut into segments of kSegJ words per lane (every level), each lane padded to whole words
// per segment, so segments are independent work items.  All integer; counts are exact by construction.
#include <cstdint>
#include <cstdlib>
#include <map>

#include "../common.h"
#include "../kernels.h"
#include "proj_dev.cuh"
#include "scan_dev.cuh"

namespace gpa {
namespace {
using namespace pj;

constexpr int kT = 256;
unsigned grid_for(uint64_t n, int n_sms, int per_sm = 16) {
  uint64_t g = (n + kT - 1) / kT;
  const uint64_t cap = (uint64_t)n_sms * per_sm;
  return (unsigned)(g < 1 ? 1 : (g > cap ? cap : g));
}

// ---------------------------------------------------------------- class structure
// A class = a run of entries with the same par_a (the left parent = the (k-2)-prefix).
// n_dev (device-sized level): the entry count lives on the device, n is its host upper bound; the
// flags are zero past the count (the scans run over n)
// class starts (entries whose left parent differs from the previous entry's; zero past the device
// count) in one launch: flag, its exclusive scan ex, bound[c] = the first entry of class c,
// bound[#classes] = |L| and *n_cls = #classes
__global__ void __launch_bounds__(sd::kScanThreads, 1) cls_scan_kernel(const uint32_t* __restrict__ par_a, uint32_t n,
                                                                       uint32_t* __restrict__ flag,
                                                                       uint32_t* __restrict__ ex,
                                                                       uint32_t* __restrict__ bound,
                                                                       uint32_t* __restrict__ n_cls,
                                                                       const uint32_t* __restrict__ n_dev,
                                                                       uint32_t* sflags, uint64_t* agg, uint64_t* inc,
                                                                       uint32_t epoch) {
  const uint32_t ne = n_dev ? min(*n_dev, n) : n;
  // n_cls[1] (max lane words, atomicMax) and n_cls[2..3] (u64 compressed words, atomicAdd) start at
  // zero for the class-table kernels that follow
  if (blockIdx.x == 0 && threadIdx.x < 3) n_cls[1 + threadIdx.x] = 0u;
  sd::scan_tile<uint32_t>(
      n,
      [&](uint32_t j) {
        const uint32_t f = j < ne && (j == 0 || par_a[j] != par_a[j - 1]);
        flag[j] = f;
        return f;
      },
      [&](uint32_t j, uint32_t e, uint32_t f) {
        ex[j] = e;
        if (f) bound[e] = j;
      },
      [&](uint32_t C) {
        bound[C] = ne;
        *n_cls = C;
      },
      sflags, agg, inc, epoch);
}

__global__ void seg_pad_kernel(Src src, const uint32_t* __restrict__ par_a, const uint32_t* __restrict__ bound,
                               const uint32_t* __restrict__ n_cls, uint32_t cmax, uint32_t nseg,
                               uint32_t* __restrict__ loc, uint32_t* __restrict__ nwc,
                               uint64_t* __restrict__ cls_words, uint32_t* __restrict__ items,
                               uint32_t* __restrict__ max_lw, uint32_t* __restrict__ len,
                               unsigned long long* __restrict__ in_words) {
  const uint32_t nc = *n_cls, n_warps = (gridDim.x * blockDim.x) >> 5;
  for (uint32_t c = (blockIdx.x * blockDim.x + threadIdx.x) >> 5; c < cmax; c += n_warps)
    seg_pad_warp(c, src, par_a, bound, nc, cmax, nseg, loc, nwc, cls_words, items, max_lw, len, in_words);
}

// warp per entry j: its vector (offset, words; entries of single-member classes get none), and
// the words past what the list build writes zeroed -- lane-interleaved lists (k >= 4): lane l's
// tail len[c][l] .. Lw_c - 1; natural-order lists (generation 3): len[c][0] .. nwc - 1
// (and, thread per (segment, class) pair, item_pair[] = the pair of every list-build item: the items
// of pair p are item_off[p] .. + items[p])
__global__ void entry_off_kernel(const uint32_t* __restrict__ flag, const uint32_t* __restrict__ ex,
                                 const uint32_t* __restrict__ bound, const uint32_t* __restrict__ nwc,
                                 const uint64_t* __restrict__ cls_base, uint32_t n, uint64_t* __restrict__ off,
                                 uint32_t* __restrict__ nw, const uint32_t* __restrict__ len, bool natural,
                                 uint32_t* __restrict__ data, const uint32_t* __restrict__ items,
                                 const uint32_t* __restrict__ item_off, uint32_t n_pairs,
                                 uint32_t* __restrict__ item_pair) {
  for (uint32_t p = blockIdx.x * blockDim.x + threadIdx.x; p < n_pairs; p += gridDim.x * blockDim.x)
    for (uint32_t i = 0; i < items[p]; ++i) item_pair[item_off[p] + i] = p;
  const uint32_t lane = threadIdx.x & 31;
  const uint32_t n_warps = (gridDim.x * blockDim.x) >> 5;
  for (uint32_t j = (blockIdx.x * blockDim.x + threadIdx.x) >> 5; j < n; j += n_warps) {
    const uint32_t c = ex[j] + flag[j] - 1;
    const uint32_t j0 = bound[c], m = bound[c + 1] - j0;
    if (m < 2) {
      if (lane == 0) {
        off[j] = 0;
        nw[j] = 0;
      }
      continue;
    }
    const uint32_t w = nwc[c];
    const uint64_t o = cls_base[c] + (uint64_t)(j - j0) * w;
    if (lane == 0) {
      nw[j] = w;
      off[j] = o;
    }
    if (natural) {
      const uint32_t i = len[(uint64_t)c * 32] + lane;
      if (i < w) data[o + i] = 0u;
    } else {
      for (uint32_t jj = len[(uint64_t)c * 32 + lane]; jj < w / 32u; ++jj) data[o + 32ull * jj + lane] = 0u;
    }
  }
}

// Hacker's Delight 7-4 "compress" (= pext): the mask-dependent shift masks, then the per-source
// part.  Right shifts by a constant are written as __umulhi(x, 2^(32-s)) and left shifts as
// multiplies so that they issue on the FMA pipe next to the LOP3s on the ALU pipe (the kernel is
// ALU-bound).  Checked bit-exact against a plain bit-by-bit pext (tests/test_host_logic.py
// ::test_compress_matches_pext runs the same sequence of operations on the host).
__device__ __forceinline__ uint32_t shr_c(uint32_t x, int s) { return __umulhi(x, 1u << (32 - s)); }
__device__ __forceinline__ uint32_t shl_c(uint32_t x, int s) { return x * (1u << s); }

__device__ __forceinline__ void hd_prep(uint32_t m, uint32_t (&mv)[5], uint32_t& m0) {
  const uint32_t m_in = m;
  uint32_t mk = shl_c(~m, 1);
#pragma unroll
  for (int i = 0; i < 5; ++i) {
    // parallel prefix XOR of mk (HD's 5 shift-xor steps) as 3-input XORs: windows 3, 9, 27, 54
    uint32_t mp = mk ^ shl_c(mk, 1) ^ shl_c(mk, 2);
    mp = mp ^ shl_c(mp, 3) ^ shl_c(mp, 6);
    mp = mp ^ shl_c(mp, 9) ^ shl_c(mp, 18);
    mp ^= shl_c(mp, 27);
    uint32_t v;  // materialised (opaque AND), so hd_apply's merge is one LOP3 on (x, mv, shifted)
    asm("and.b32 %0, %1, %2;" : "=r"(v) : "r"(mp), "r"(m));
    mv[i] = v;
    m = (m ^ v) | shr_c(v, 1 << i);
    mk &= ~mp;
  }
  asm("lop3.b32 %0, %1, %2, 0, 0x30;" : "=r"(m0) : "r"(m_in), "r"(mv[0]));  // m & ~mv0: bits kept by stage 0
}
// pext(x, m) given m's shift masks (x need not be pre-masked: stage 0 keeps x & m0 and moves x & mv0)
// (each stage is two LOP3 -- the moving bits, then keep-or-moved in one 3-input op -- and one
// IMAD.HI; written as PTX lop3 so that the compiler cannot split the merge into AND + OR)
__device__ __forceinline__ uint32_t hd_apply(uint32_t x, uint32_t m0, const uint32_t (&mv)[5]) {
  uint32_t t, y;
  asm("and.b32 %0, %1, %2;" : "=r"(t) : "r"(x), "r"(mv[0]));
  asm("lop3.b32 %0, %1, %2, %3, 0xEA;" : "=r"(y) : "r"(x), "r"(m0), "r"(shr_c(t, 1)));  // (x & m0) | ts
#pragma unroll
  for (int i = 1; i < 5; ++i) {
    asm("and.b32 %0, %1, %2;" : "=r"(t) : "r"(y), "r"(mv[i]));
    asm("lop3.b32 %0, %1, %2, %3, 0xBA;" : "=r"(y) : "r"(y), "r"(mv[i]), "r"(shr_c(t, 1 << i)));  // (y & ~mv) | ts
  }
  return y;
}

// One item of pext_kernel for a group of nm <= G members (G = 2, 3, 4, 6, 8: the unrolled width, so
// a class of 2 members does not pay for 8): lane l walks its mask words [ja, jb) and appends, for
// every member, pext(source word, mask word) to the member's lane-l stream -- a 32-bit
// accumulator, whole words stored as they fill, the last partial word at the segment's end.
// The bit count per step is the mask's, the same for every member, so the fill level and the
// output position are shared; the append is one 32x32->64 multiply by 2^fill.  The next step's
// mask and source words are loaded one step ahead.
// base + idx words as one IMAD.WIDE.U32 on the FMA pipe: the scale (4) comes from a kernel
// parameter, otherwise ptxas turns the multiply by a constant 4 into LEA + LEA.HI.X on the ALU pipe
__device__ __forceinline__ const uint32_t* addr_of(const uint32_t* base, uint32_t idx, uint32_t wbytes) {
  const uint32_t* r;
  asm("mad.wide.u32 %0, %1, %2, %3;" : "=l"(r) : "r"(idx), "r"(wbytes), "l"(base));
  return r;
}

// base + 4 idx in one IMAD.WIDE (immediate scale: ptxas keeps the 64-bit addend in the multiply-add)
__device__ __forceinline__ const uint32_t* addr4(const uint32_t* base, uint32_t idx) {
  const uint32_t* r;
  asm("mad.wide.u32 %0, %1, 4, %2;" : "=l"(r) : "r"(idx), "l"(base));
  return r;
}

template <uint32_t G, bool SPARSE>
__device__ __forceinline__ void pext_item(const uint32_t* __restrict__ mp, const uint32_t* __restrict__ sbase,
                                          const uint32_t (&so)[kMemberGroup], const uint32_t* __restrict__ s_oo,
                                          uint32_t nm, uint32_t ja, uint32_t jb, uint32_t oj,
                                          uint32_t* __restrict__ data, uint32_t wbytes) {
  // member q's word j of this lane: cur + so[q] with cur = sbase + 32 j (one 64-bit step per j, then
  // one IMAD.WIDE per member); output base offsets in shared memory (read only when a word fills)
  uint32_t acc[G], xn[G];
  uint32_t nb = 0;
  mp += 32u * ja;
  const uint32_t* cur = sbase + 32u * ja;
  uint32_t mn = __ldg(mp);
#pragma unroll
  for (uint32_t q = 0; q < G; ++q) {
    acc[q] = 0;
    xn[q] = __ldg(addr_of(cur, so[q], wbytes));
  }
  for (uint32_t j = ja; j < jb; ++j) {
    const uint32_t mw = mn;
    uint32_t x[G];
#pragma unroll
    for (uint32_t q = 0; q < G; ++q) x[q] = xn[q];
    const uint32_t step = j + 1 < jb ? 32u : 0u;
    mp += step;
    cur += step;
    mn = __ldg(mp);
#pragma unroll
    for (uint32_t q = 0; q < G; ++q) xn[q] = __ldg(addr_of(cur, so[q], wbytes));
    const uint32_t pw = 1u << nb;
    const uint32_t c = __popc(mw);
    nb += c;
    uint32_t y[G];
    if constexpr (SPARSE) {
      // sparse masks (bitset rows, ~5 % set): the mask's trailing ones stay in place; every further
      // set bit p lands at position i = its rank: bit i of (x >> (p - i)), the shift as an IMAD.HI by
      // 2^(32 - (p - i)) (p - i >= 1 past the trailing ones) shared by the group -- per member one
      // IMAD.HI + one LOP3 per set bit; the loop runs to the warp's largest count
      const uint32_t i0 = mw == 0xffffffffu ? 32u : (uint32_t)__ffs(~mw) - 1u;
      const uint32_t idm = i0 >= 32 ? 0xffffffffu : (1u << i0) - 1u;
#pragma unroll
      for (uint32_t q = 0; q < G; ++q) y[q] = x[q] & idm;
      uint32_t mm = mw & ~idm, i = i0;
      const uint32_t T = __reduce_max_sync(0xffffffffu, c - min(i0, c));
      for (uint32_t t = 0; t < T; ++t) {
        const bool has = mm != 0;
        const uint32_t pbit = has ? (uint32_t)__ffs(mm) - 1u : 0u;
        mm &= mm - 1u;
        const uint32_t M = has ? 1u << (32u - (pbit - i)) : 0u;
        const uint32_t bi = has ? 1u << i : 0u;
#pragma unroll
        for (uint32_t q = 0; q < G; ++q) {
          uint32_t r;
          asm("lop3.b32 %0, %1, %2, %3, 0xF8;" : "=r"(r) : "r"(y[q]), "r"(__umulhi(x[q], M)), "r"(bi));  // y | (t & bi)
          y[q] = r;
        }
        i += has ? 1u : 0u;
      }
    } else {
      uint32_t mv[5], m0;
      hd_prep(mw, mv, m0);
#pragma unroll
      for (uint32_t q = 0; q < G; ++q) y[q] = hd_apply(x[q], m0, mv);
    }
#pragma unroll
    for (uint32_t q = 0; q < G; ++q) {
      // append at bit nb: one 32x32->64 multiply by 2^nb (FMA pipe); the low half is disjoint from
      // the bits already in acc, so the OR is an add (FMA pipe as well); x[q] keeps the carry
      uint64_t v;
      asm("mul.wide.u32 %0, %1, %2;" : "=l"(v) : "r"(y[q]), "r"(pw));
      asm("mad.lo.u32 %0, %1, 1, %0;" : "+r"(acc[q]) : "r"((uint32_t)v));
      x[q] = (uint32_t)(v >> 32);
    }
    if (nb >= 32) {
#pragma unroll
      for (uint32_t q = 0; q < G; ++q) {
        if (q < nm) data[s_oo[q] + 32u * oj] = acc[q];
        acc[q] = x[q];
      }
      ++oj;
      nb -= 32;
    }
  }
  if (nb) {
#pragma unroll
    for (uint32_t q = 0; q < G; ++q)
      if (q < nm) data[s_oo[q] + 32u * oj] = acc[q];
  }
}

// ---------------------------------------------------------------- generation 3: bit gather
// Generation 3's masks are bitset rows (~5 % set): instead of compressing every word per lane,
// the warp gathers the ~C set bits of a 32-word chunk (row words 32 j .. 32 j + 31, one per lane)
// in ceil(C / 32) ballots: lane l stages (l, bit) of its set bits in shared memory at its rank
// (warp scan of the popcounts), then lane r of ballot t takes set bit 32 t + r, fetches the
// member's word from its owner lane (shfl) and the ballot packs 32 of those bits into one output
// word.  A member's list is the concatenation of these words (each chunk padded to whole words;
// natural order, common to the class -- the next generation views it as 32 lane streams).
// Work ~ output words, not input words.  (seg3 / cls3: sizes; pext3: the lists.)

__global__ void seg3_kernel(const uint32_t* __restrict__ rows, uint64_t pitch, const uint32_t* __restrict__ par_a,
                            const uint32_t* __restrict__ bound, const uint32_t* __restrict__ n_cls, uint32_t cmax,
                            uint32_t n_pairs, uint32_t* __restrict__ w3, unsigned long long* __restrict__ in_words) {
  const uint32_t nc = *n_cls, n_warps = (gridDim.x * blockDim.x) >> 5;
  for (uint32_t p = (blockIdx.x * blockDim.x + threadIdx.x) >> 5; p < n_pairs; p += n_warps)
    seg3_warp(p, rows, pitch, par_a, bound, nc, cmax, w3, in_words);
}

__global__ void cls3_pad_kernel(const uint32_t* __restrict__ w3, const uint32_t* __restrict__ bound,
                                const uint32_t* __restrict__ n_cls, uint32_t cmax, uint32_t nseg,
                                uint32_t* __restrict__ loc3, uint32_t* __restrict__ nwc,
                                uint64_t* __restrict__ cls_words, uint32_t* __restrict__ items,
                                uint32_t* __restrict__ max_lw, uint32_t* __restrict__ len) {
  const uint32_t C = *n_cls;
  for (uint32_t c = blockIdx.x * blockDim.x + threadIdx.x; c < cmax; c += gridDim.x * blockDim.x)
    cls3_pad_thread(c, w3, bound, C, cmax, nseg, loc3, nwc, cls_words, items, max_lw, len);
}

// pext3 per-warp shared memory: two stages of the group's member words of one 64-word chunk (the
// chunk being packed, the next one arriving by cp.async) and the chunk's staged set bits.
constexpr uint32_t kP3Warps = 4;
constexpr uint32_t kP3Blocks = 6;     // blocks/SM (shared memory: 4 x 9.3 KB per block; 4 x 6 measured 2.5 % faster than 8 x 3 and 2 x 12)
constexpr uint32_t kP3Chunk = 64;     // mask words per chunk: two per lane
constexpr uint32_t kP3Pos = 448;      // staged set bits per pass (a chunk holds up to 2,048)
constexpr uint16_t kP3None = 32;      // staged code of "no bit": word 0, shift 32 -> empty mask
struct P3Warp {
  uint32_t xs[2][kG3Group][kP3Chunk];  // member q's words of the chunk
  uint16_t pos[32 + kP3Pos + 32];      // a pass of the chunk's set bits in rank order: word << 6 | bit
  uint32_t oo[kG3Group];               // member list: word offset in data
};

__device__ __forceinline__ void cp_async16(uint32_t dst, const void* src) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(dst), "l"(src) : "memory");
}

// One item of pext3_kernel: a group of nm <= G members of a class over the mask segment's chunks
// [ca, cb) (64 words each).  Per chunk: lane l holds mask words 2l, 2l + 1; a warp scan of their
// popcounts ranks the chunk's C set bits, which are staged in rank order; output words are packed
// by ballots over ranks.  Set bits carry across chunks: the word of a chunk's last pend (< 32) bits
// is gathered at once (lanes >= pend vote 0) and stays in its output slot, and the next chunk's
// first ballot ORs its bits in at lanes pend .. 31 -- the segment's bits are packed densely,
// ceil(bits / 32) words (seg3_warp), and no chunk's words are needed after the chunk.  Per member
// and output word: LDS + LOP3 (-> predicate) + VOTE + LOP3 (into lane slot's register).
template <uint32_t G>
__device__ __forceinline__ void pext3_item(P3Warp& w, const uint32_t* __restrict__ mrow,
                                           const uint32_t* __restrict__ rows, uint32_t so_l, uint32_t nm,
                                           uint32_t ca, uint32_t cb, uint32_t ow0, uint32_t* __restrict__ data) {
  static_assert(G % 2 == 0 && G <= kG3Group, "members are staged two per cp.async instruction");
  const uint32_t lane = threadIdx.x & 31;
  // lane l stages 16 bytes of member 2i + (l >> 4): words 4 (l & 15) .. + 3 of the chunk
  uint32_t my_so[G / 2];
#pragma unroll
  for (uint32_t i = 0; i < G / 2; ++i) my_so[i] = __shfl_sync(0xffffffffu, so_l, 2 * i + (lane >> 4)) + 4u * (lane & 15u);
  const uint32_t xs_lane = (uint32_t)__cvta_generic_to_shared(&w.xs[0][lane >> 4][4u * (lane & 15u)]);
  auto stage = [&](uint32_t c, uint32_t st) {
    const uint32_t* cur = rows + (uint64_t)c * kP3Chunk;
    const uint32_t dst = xs_lane + st * (uint32_t)sizeof(w.xs[0]);
#pragma unroll
    for (uint32_t i = 0; i < G / 2; ++i) cp_async16(dst + i * 2u * kP3Chunk * 4u, addr4(cur, my_so[i]));
    asm volatile("cp.async.commit_group;" ::: "memory");
  };
  uint32_t keep[G];
#pragma unroll
  for (uint32_t q = 0; q < G; ++q) keep[q] = 0;
  uint32_t wc = 0;    // whole words packed in this segment (warp-uniform)
  uint32_t pend = 0;  // set bits in the open word (slot wc & 31), < 32
  stage(ca, 0);
  const uint2* mp = reinterpret_cast<const uint2*>(mrow) + lane;
  uint2 mn = __ldg(mp + (uint64_t)ca * (kP3Chunk / 2));
  for (uint32_t c = ca; c < cb; ++c) {
    const uint32_t st = (c - ca) & 1u;
    const uint2 m = mn;
    asm volatile("cp.async.wait_group 0;" ::: "memory");
    __syncwarp();  // chunk c's member words visible to the warp; chunk c - 1's reads are done
    if (c + 1 < cb) {
      stage(c + 1, st ^ 1u);
      mn = __ldg(mp + (uint64_t)(c + 1) * (kP3Chunk / 2));
    }
    // ranks of this lane's set bits: warp scan of the popcounts
    const uint32_t cnt = __popc(m.x) + __popc(m.y);
    uint32_t o = cnt;
#pragma unroll
    for (uint32_t d = 1; d < 32; d <<= 1) {
      const uint32_t t = __shfl_up_sync(0xffffffffu, o, d);
      if (lane >= d) o += t;
    }
    const uint32_t Call = __shfl_sync(0xffffffffu, o, 31);
    // the chunk's set bits in passes of at most kP3Pos ranks (one pass below 22 % density).  A pass
    // stages pos[pend + r] = the code (word << 6 | bit) of its rank r, with kP3None -- bit 32, i.e.
    // an empty bit mask -- in the pend slots before and the 32 after, so that ballot t reads
    // pos[32 t + lane] with no range test (the carried lanes and the tail vote 0)
    for (uint32_t lo = 0; lo < Call; lo += kP3Pos) {
      const uint32_t C = min(Call - lo, kP3Pos);
      {
        // 32-bit walks (a 64-bit one costs ~2.5x the instructions per set bit)
        const uint32_t code0 = lane * 128u;   // word 2 lane, bit 0
        if (lane < pend) w.pos[lane] = kP3None;
        w.pos[pend + C + lane] = kP3None;
        if (Call <= kP3Pos) {
          uint16_t* pp = &w.pos[pend + o - cnt];
          for (uint32_t mm = m.x; mm; mm &= mm - 1u) *pp++ = (uint16_t)(code0 + (uint32_t)(__ffs(mm) - 1));
          for (uint32_t mm = m.y; mm; mm &= mm - 1u) *pp++ = (uint16_t)(code0 + 63u + (uint32_t)__ffs(mm));
        } else {   // dense chunk: only the ranks of this pass
          uint32_t r = o - cnt - lo;
          for (uint32_t mm = m.x; mm; mm &= mm - 1u, ++r)
            if (r < C) w.pos[pend + r] = (uint16_t)(code0 + (uint32_t)(__ffs(mm) - 1));
          for (uint32_t mm = m.y; mm; mm &= mm - 1u, ++r)
            if (r < C) w.pos[pend + r] = (uint16_t)(code0 + 63u + (uint32_t)__ffs(mm));
        }
      }
      __syncwarp();
      const uint32_t tot = pend + C, full = tot >> 5;
      const uint32_t nb = full + ((tot & 31u) ? 1u : 0u);
      const uint32_t* xst = &w.xs[st][0][0];
      const uint16_t* pl = &w.pos[lane];
      for (uint32_t t = 0; t < nb; ++t) {
        // lane r takes the pass' set bit of rank 32 t + r - pend
        const uint32_t code = pl[32u * t];
        uint32_t bm;
        asm("shl.b32 %0, 1, %1;" : "=r"(bm) : "r"(code & 63u));   // bit 32 (kP3None): 0
        const uint32_t* xb = xst + (code >> 6);
        const uint32_t sel = lane == (wc & 31u) ? 0xffffffffu : 0u;
#pragma unroll
        for (uint32_t q = 0; q < G; ++q) {
          const uint32_t b = __ballot_sync(0xffffffffu, (xb[q * kP3Chunk] & bm) != 0u);
          uint32_t r;
          asm("lop3.b32 %0, %1, %2, %3, 0xF8;" : "=r"(r) : "r"(keep[q]), "r"(b), "r"(sel));  // keep | (b & sel)
          keep[q] = r;
        }
        if (t < full) {  // a whole word: the next slot; 32 slots full -> one coalesced store per member
          if ((++wc & 31u) == 0u) {
#pragma unroll
            for (uint32_t q = 0; q < G; ++q) {
              if (q < nm) data[w.oo[q] + ow0 + (wc - 32u) + lane] = keep[q];
              keep[q] = 0;
            }
          }
        }
      }
      pend = tot & 31u;
      __syncwarp();  // pos (and, after the chunk, this stage) are rewritten next
    }
  }
  // the last whole words and the open partial word (its high bits zero)
  const uint32_t left = (wc & 31u) + (pend ? 1u : 0u);
  if (lane < left) {
#pragma unroll
    for (uint32_t q = 0; q < G; ++q)
      if (q < nm) data[w.oo[q] + ow0 + (wc & ~31u) + lane] = keep[q];
  }
}

__global__ void __launch_bounds__(kP3Warps * 32, kP3Blocks) pext3_kernel(const uint32_t* __restrict__ rows, uint64_t pitch,
                                                                 const uint32_t* __restrict__ par_a,
                                                                 const uint32_t* __restrict__ par_b,
                                                                 const uint32_t* __restrict__ bound, uint32_t cmax,
                                                                 const uint32_t* __restrict__ item_pair,
                                                                 const uint32_t* __restrict__ item_off, uint32_t T,
                                                                 const uint32_t* __restrict__ loc3,
                                                                 const uint64_t* __restrict__ off,
                                                                 uint32_t* __restrict__ data) {
  extern __shared__ __align__(16) unsigned char p3_smem[];
  P3Warp& w = reinterpret_cast<P3Warp*>(p3_smem)[threadIdx.x >> 5];
  const uint32_t lane = threadIdx.x & 31;
  const uint32_t it = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  if (it >= T) return;
  const uint32_t p = item_pair[it];
  const uint32_t c = p % cmax, s = p / cmax;
  const uint32_t j0 = bound[c], m = bound[c + 1] - j0;
  const uint32_t g = it - item_off[p];
  const uint32_t first = j0 + g * kG3Group;
  const uint32_t nm = min(kG3Group, m - g * kG3Group);
  uint32_t ja, jb;   // the segment in 32-word steps (a multiple of 2: pitch is a multiple of 1,024 words)
  seg_range((uint32_t)(pitch / 32), s, ja, jb);
  if (ja >= jb) return;
  // member row offsets (slots >= nm shadow member 0: staged and gathered, never stored)
  const uint32_t e = first + (lane < nm ? lane : 0u);
  const uint32_t so_l = (uint32_t)((uint64_t)par_b[e] * pitch);
  if (lane < kG3Group) w.oo[lane] = (uint32_t)off[e];
  __syncwarp();
  const uint32_t* mrow = rows + (uint64_t)par_a[j0] * pitch;
  const uint32_t ow0 = loc3[p];
  const uint32_t ca = ja / 2, cb = jb / 2;
  if (nm <= 4)
    pext3_item<4>(w, mrow, rows, so_l, nm, ca, cb, ow0, data);
  else if (nm <= 8)
    pext3_item<8>(w, mrow, rows, so_l, nm, ca, cb, ow0, data);
  else if (nm <= 12)
    pext3_item<12>(w, mrow, rows, so_l, nm, ca, cb, ow0, data);
  else
    pext3_item<16>(w, mrow, rows, so_l, nm, ca, cb, ow0, data);
}

// Warp per item = (pair p = (segment, class), group of <= kMemberGroup members: full groups of 8,
// the remainder in the class' last group).  Items run pair-major = segment-major, so the warps in
// flight share the same bitset segments in L2.
constexpr int kPextT = 128;   // pext_kernel block (8 blocks/SM: the same 32 warps, finer scheduling)
__global__ void __launch_bounds__(kPextT, 8) pext_kernel(Src src, const uint32_t* __restrict__ par_a,
                                                     const uint32_t* __restrict__ par_b,
                                                     const uint32_t* __restrict__ bound, uint32_t cmax,
                                                     const uint32_t* __restrict__ item_pair,
                                                     const uint32_t* __restrict__ item_off,
                                                     uint32_t T, const uint32_t* __restrict__ loc,
                                                     const uint64_t* __restrict__ off, uint32_t* __restrict__ data,
                                                     uint32_t wbytes) {
  const uint32_t lane = threadIdx.x & 31;
  const uint32_t it = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  if (it >= T) return;
  const uint32_t* base = src.rows ? src.rows : src.data;
  {
    const uint32_t p = item_pair[it];
    const uint32_t c = p % cmax, s = p / cmax;
    const uint32_t j0 = bound[c], m = bound[c + 1] - j0;
    const uint32_t groups = (m + kMemberGroup - 1) / kMemberGroup;
    const uint32_t g = it - item_off[p];
    (void)groups;
    const uint32_t first = j0 + g * kMemberGroup;  // full groups of 8, the remainder in the last
    const uint32_t nm = min(kMemberGroup, m - g * kMemberGroup);
    const VecRef mk = src.vec(par_a[j0]);
    uint32_t ja, jb;
    seg_range(mk.lw, s, ja, jb);
    if (ja >= jb) return;
    __shared__ uint32_t s_oo[kPextT / 32][kMemberGroup];
    uint32_t* oo = s_oo[threadIdx.x >> 5];
    uint32_t so[kMemberGroup];
#pragma unroll
    for (uint32_t q = 0; q < kMemberGroup; ++q) {
      const uint32_t e = first + (q < nm ? q : 0);  // surplus slots shadow member 0 (not stored)
      so[q] = (uint32_t)(src.vec(par_b[e]).p - base);
      if (lane == q) oo[q] = (uint32_t)off[e] + 0u;
    }
    __syncwarp();
    const uint32_t oj = loc[(uint64_t)p * 32 + lane];
    const uint32_t* mp = mk.p + lane;
    if (src.rows) {  // generation 3: sparse bitset rows as masks
      if (nm <= 2)
        pext_item<2, true>(mp, base + lane, so, oo, nm, ja, jb, oj, data + lane, wbytes);
      else if (nm <= 4)
        pext_item<4, true>(mp, base + lane, so, oo, nm, ja, jb, oj, data + lane, wbytes);
      else
        pext_item<8, true>(mp, base + lane, so, oo, nm, ja, jb, oj, data + lane, wbytes);
    } else if (nm <= 2) {
      pext_item<2, false>(mp, base + lane, so, oo, nm, ja, jb, oj, data + lane, wbytes);
    } else if (nm == 3) {
      pext_item<3, false>(mp, base + lane, so, oo, nm, ja, jb, oj, data + lane, wbytes);
    } else if (nm <= 4) {
      pext_item<4, false>(mp, base + lane, so, oo, nm, ja, jb, oj, data + lane, wbytes);
    } else if (nm <= 6) {
      pext_item<6, false>(mp, base + lane, so, oo, nm, ja, jb, oj, data + lane, wbytes);
    } else {
      pext_item<8, false>(mp, base + lane, so, oo, nm, ja, jb, oj, data + lane, wbytes);
    }
  }
}

// ---------------------------------------------------------------- counting
// WARP = false: CTA per group g (left parent x = gpar[g]), its warps striding over 256-word chunks
// of the class lists, one atomic per (warp, sibling) -- long lists (generation 3); WARP = true:
// one warp per group walking the whole list, plain stores -- short lists (deep generations, where
// a CTA per group would leave most of its warps idle).  Siblings in batches of 32 (lane j
// accumulates sibling j); two siblings share one packed redux.sync (per-chunk warp sums
// <= 32 x 8 x 32 < 2^16).
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
      if constexpr (WARP) {   // short lists, few siblings: two at a time
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
        continue;
      }
      // long lists: 4 siblings per step, their 8 loads issued together, then two packed reductions
      for (uint32_t i = 0; i < nb; i += 4) {
        uint4 ya[4], yb[4];
#pragma unroll
        for (uint32_t q = 0; q < 4; ++q) {
          const uint64_t yo = __shfl_sync(0xffffffffu, my_off, (i + q) & 31u);
          const bool ok = i + q < nb;
          const uint32_t* Y = data + yo;
          ya[q] = ok && h0 ? *reinterpret_cast<const uint4*>(Y + w0) : make_uint4(0, 0, 0, 0);
          yb[q] = ok && h1 ? *reinterpret_cast<const uint4*>(Y + w1) : make_uint4(0, 0, 0, 0);
        }
#pragma unroll
        for (uint32_t pq = 0; pq < 4; pq += 2) {
          if (i + pq >= nb) break;   // warp-uniform
          uint32_t c = 0;
#pragma unroll
          for (uint32_t q = 0; q < 2; ++q) {
            const uint4 y0 = ya[pq + q], y1 = yb[pq + q];
            const uint32_t v = __popc(x0.x & y0.x) + __popc(x0.y & y0.y) + __popc(x0.z & y0.z) +
                               __popc(x0.w & y0.w) + __popc(x1.x & y1.x) + __popc(x1.y & y1.y) +
                               __popc(x1.z & y1.z) + __popc(x1.w & y1.w);
            c |= v << (16 * q);
          }
          c = __reduce_add_sync(0xffffffffu, c);
          if (lane == i + pq) acc += c & 0xffffu;
          if (lane == i + pq + 1) acc += c >> 16;
        }
      }
    }
    if (WARP) {
      if (lane < nb) counts[b0 + lane] = acc;
    } else if (lane < nb && acc) {
      atomicAdd(&counts[b0 + lane], acc);
    }
  }
}



// generation 3 by bit gather (pext3_kernel); GPA_PROJ_K3_PEXT=1 keeps the set-bit-walk pext (comparisons)
bool gather3() {
  static const bool v = [] {
    const char* e = getenv("GPA_PROJ_K3_PEXT");
    return !(e && atoi(e) != 0);
  }();
  return v;
}

// per-thread, per-device persistent workspace (grow-only): the class tables of proj_build and the
// two generations of lists
struct ProjWork {
  PBuf<uint32_t> flag, ex, bound, small, words, loc, items, item_off, item_pair, nwc, len;
  PBuf<uint64_t> cls_words, cls_base, tot;
  ScanState scan;      // scan status words of its own: proj_build_begin runs beside the join's scans
  DeviceProj lists[2];
};
ProjWork& work_for(int device) {
  thread_local std::map<int, ProjWork> w;
  return w[device];
}

}  // namespace

DeviceProj* proj_lists(int device) { return work_for(device).lists; }

namespace {
Src make_src(const ProjPending& pp) {
  Src src{};
  if (!pp.prev) {
    src.rows = pp.rows;
    src.pitch = pp.pitch;
  } else {
    src.data = pp.prev->data.p;
    src.off = pp.prev->off.p;
    src.nw = pp.prev->nw.p;
  }
  return src;
}
}  // namespace

bool proj_build_begin(uint32_t n, const uint32_t* par_a, const uint32_t* par_b, const DeviceProj* prev,
                      const uint32_t* rows, uint64_t pitch_words, uint32_t n_rows, DeviceScratch& scratch, int n_sms,
                      cudaStream_t s, ProjPending& pp, const uint32_t* n_dev, uint32_t* d_block, cudaStream_t pre,
                      cudaEvent_t fork) {
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
  const uint64_t lw_max = prev ? prev->max_lw : pitch_words / 32;
  const uint32_t nseg = (uint32_t)std::max<uint64_t>(1, (lw_max + kSegJ - 1) / kSegJ);
  // 32-bit word offsets inside pext_kernel
  // pext_kernel addresses sources with 32-bit word offsets, its tables with 31-bit indices: beyond
  // that the caller uses complete intersection
  if (!prev && (uint64_t)n_rows * pitch_words >= (1ull << 32)) return false;
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
  W.small.ensure(4);   // zeroed by cls_scan_kernel
  W.tot.ensure(2);
  // counters and totals in the caller's size block (one host read per generation) or our own
  uint32_t* const small = d_block ? d_block + 6 : W.small.p;
  uint64_t* const tot = d_block ? reinterpret_cast<uint64_t*>(d_block + 2) : W.tot.p;
  {
    const uint32_t tiles = scan_tiles(n);
    const uint32_t ep = scan_epoch(W.scan, tiles, pre ? pre : s);
    cls_scan_kernel<<<tiles, sd::kScanThreads, 0, pre ? pre : s>>>(par_a, n, W.flag.p, W.ex.p, W.bound.p, small,
                                                                   n_dev, W.scan.flags.p, W.scan.agg.p, W.scan.inc.p,
                                                                   ep);
    note_launch();
  }
  if (pre) {   // the rest of the class tables on s, after the class scan on pre
    GPA_CUDA(cudaEventRecord(fork, pre));
    GPA_CUDA(cudaStreamWaitEvent(s, fork, 0));
  }
  pp.flag = W.flag.p;
  pp.ex = W.ex.p;
  pp.bound = W.bound.p;
  W.words.ensure((size_t)n_pairs * 32);
  W.loc.ensure((size_t)n_pairs * 32);
  W.items.ensure(n_pairs);
  W.item_off.ensure(n_pairs);
  W.nwc.ensure(cmax);
  W.cls_words.ensure(cmax);
  W.cls_base.ensure(cmax);
  W.len.ensure((size_t)cmax * 32);
  const unsigned wpb = kT / 32;
  if (!prev && gather3()) {  // generation 3: bit gather (pext3_kernel), natural-order lists
    { seg3_kernel<<<grid_for(32ull * n_pairs, n_sms), kT, 0, s>>>(rows, pitch_words, par_a, W.bound.p, small, cmax, n_pairs,
          W.words.p, reinterpret_cast<unsigned long long*>(small + 2)); note_launch(); }
    { cls3_pad_kernel<<<grid_for(cmax, n_sms), kT, 0, s>>>(W.words.p, W.bound.p, small, cmax, nseg, W.loc.p,
          W.nwc.p, W.cls_words.p, W.items.p, small + 1, W.len.p); note_launch(); }
  } else {
    { seg_pad_kernel<<<grid_for(32ull * cmax, n_sms), kT, 0, s>>>(
          src, par_a, W.bound.p, small, cmax, nseg, W.loc.p, W.nwc.p, W.cls_words.p, W.items.p, small + 1, W.len.p,
          reinterpret_cast<unsigned long long*>(small + 2));
      note_launch(); }
  }
  // tot = {pext items, list words}: the totals of the two scans
  scan_excl_dual(W.items.p, W.item_off.p, n_pairs, tot, W.cls_words.p, W.cls_base.p, cmax, tot + 1, W.scan, s);
  GPA_CUDA(cudaGetLastError());
  pp.d_tot = tot;
  pp.d_small = small;
  return true;
}

bool proj_build_finish(const ProjPending& pp, const uint64_t T[2], const uint32_t sm[4], DeviceProj& out, int n_sms,
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
  try {
    out.data.ensure(T[1]);
  } catch (const Error& e) {
    if (e.status != GPA_ERR_OOM) throw;
    return false;  // caller falls back to complete intersection
  }
  ProjWork& W = work_for(pp.device);
  const Src src = make_src(pp);
  out.off.ensure(n);
  out.nw.ensure(n);
  out.words = T[1];
  out.max_lw = sm[1];
  out.in_words = (uint64_t)sm[2] | ((uint64_t)sm[3] << 32);
  // offsets, the zero tails of lanes shorter than their class' Lw (the list build writes the rest)
  // and the item -> pair map of the list build
  W.item_pair.ensure(std::max<uint64_t>(T[0], 1));
  { entry_off_kernel<<<grid_for(std::max<uint64_t>(32ull * n, pp.n_pairs), n_sms), kT, 0, s>>>(
        W.flag.p, W.ex.p, W.bound.p, W.nwc.p, W.cls_base.p, n, out.off.p, out.nw.p, W.len.p, !pp.prev && gather3(),
        out.data.p, W.items.p, W.item_off.p, T[0] ? pp.n_pairs : 0u, W.item_pair.p);
    note_launch(); }
  if (ev_build) GPA_CUDA(cudaEventRecord(ev_build, s));  // start of the list build proper
  if (T[0]) {
    const uint64_t blocks = (T[0] + kPextT / 32 - 1) / (kPextT / 32);
    if (!pp.prev && gather3()) {
      const int smem = (int)(kP3Warps * sizeof(P3Warp));
      ensure_smem_attr((const void*)pext3_kernel, smem);
      pext3_kernel<<<(unsigned)((T[0] + kP3Warps - 1) / kP3Warps), kP3Warps * 32, smem, s>>>(
          pp.rows, pp.pitch, pp.par_a, pp.par_b, W.bound.p, pp.cmax, W.item_pair.p, W.item_off.p, (uint32_t)T[0],
          W.loc.p, out.off.p, out.data.p);
      note_launch();
    } else
      { pext_kernel<<<(unsigned)blocks, kPextT, 0, s>>>(src, pp.par_a, pp.par_b, W.bound.p, pp.cmax, W.item_pair.p,
                                                    W.item_off.p, (uint32_t)T[0], W.loc.p, out.off.p, out.data.p, 4u);
        note_launch(); }
  }
  GPA_CUDA(cudaGetLastError());
  return true;
}

bool proj_build(uint32_t n, const uint32_t* par_a, const uint32_t* par_b, const DeviceProj* prev,
                const uint32_t* rows, uint64_t pitch_words, uint32_t n_rows, DeviceProj& out, DeviceScratch& scratch,
                int n_sms, cudaStream_t s, cudaEvent_t ev_build) {
  ProjPending pp;
  if (!proj_build_begin(n, par_a, par_b, prev, rows, pitch_words, n_rows, scratch, n_sms, s, pp, nullptr)) return false;
  uint64_t T[2] = {0, 0};
  uint32_t sm[4] = {0, 0, 0, 0};
  if (n) {
    GPA_CUDA(cudaMemcpyAsync(T, pp.d_tot, sizeof(T), cudaMemcpyDeviceToHost, s));
    GPA_CUDA(cudaMemcpyAsync(sm, pp.d_small, sizeof(sm), cudaMemcpyDeviceToHost, s));
    stream_wait(s);
  }
  return proj_build_finish(pp, T, sm, out, n_sms, s, ev_build);
}

bool count_proj_stores_all(const DeviceProj& P) { return (uint64_t)P.max_lw * 32 <= 8192; }

void launch_count_proj(const DeviceProj& P, const uint32_t* gpar, const uint32_t* ext_off, const uint32_t* eidx,
                       uint32_t G, uint32_t* counts, cudaStream_t s) {
  if (G == 0) return;
  if (count_proj_stores_all(P))
    { count_proj_kernel<true><<<(G + kT / 32 - 1) / (kT / 32), kT, 0, s>>>(P.data.p, P.off.p, P.nw.p, gpar, ext_off,
                                                                          eidx, counts, G); note_launch(); }
  else
    { count_proj_kernel<false><<<G, kT, 0, s>>>(P.data.p, P.off.p, P.nw.p, gpar, ext_off, eidx, counts, G);
      note_launch(); }
  GPA_CUDA(cudaGetLastError());
}

}  // namespace gpa
