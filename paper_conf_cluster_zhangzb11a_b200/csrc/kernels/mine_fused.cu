// The whole level-wise loop in ONE cooperative launch, for problems whose L_1 bitset sits in L2
// (sm_100a).  SURVEY.md §8(f) f1: "a fully device-resident level loop (CUDA graph or persistent
// kernel, no per-level D2H)".
//
// Small databases (the chess-, mushroom-, accidents-shaped and T40I10D100K configurations: <= 1,024 frequent
// items, a few MB of bitset) are latency-bound: the multi-kernel path spends ~30 launches and a
// host synchronisation per generation on a few microseconds of counting.  Here every generation is
// a sequence of grid-wide phases separated by grid.sync() -- no launch, no host round trip:
//
//   count    supp(c) = popc(AND of the k rows of c) -- the paper's complete intersection (P18@394),
//            a warp per (prefix group, <= 32 extensions): the (k-1)-row prefix AND per 32-word
//            chunk in registers, one AND + POPC per extension word, per-lane accumulators reduced
//            once per batch (redux.sync)
//   threshold L_k = { c : count >= theta } (P13@474, ">=" per DESIGN.md Q1): flag, grid scan,
//            scatter of the rows in candidate (= lexicographic) order, the frequent itemsets and
//            supports appended to the output arena in original item ids
//   join     C_{k+1} = join of run siblings + prune by a hash set of L_k (P13@1006-1270, P13@178),
//            grouped by k-prefix: run starts, grid scan, run bounds, hash insert, survivor counts,
//            grid scans of the counts and of the non-empty groups, emit
//
// Termination when L_k or C_{k+1} is empty (P13@652) or after max_k.  Capacities are fixed at
// launch; an overflow sets a status bit and the host reruns the problem on the multi-kernel path
// (never a CPU path).  Integer only; the same sets and counts as every other path.
#include <cooperative_groups.h>
#include <algorithm>
#include <map>
#include <vector>
#include <cstdint>
#include <cstdlib>

#include "../common.h"
#include "../kernels.h"
#include "level_dev.cuh"

namespace cg = cooperative_groups;

namespace gpa {
namespace {

constexpr int kFT = 1024;                // threads per CTA (one CTA per SM: cheap grid syncs)
constexpr uint32_t kFusedStageWords = 2048;   // staged tile words per CTA (tile batches of 2,048 / (32 |L_1|) tiles; measured 1,024 / 2,048 / 4,096 / 8,192 / 32,768: 2,048 best overall)
constexpr uint32_t kNoSlot = 0xffffffffu, kClaimed = 0xfffffffeu;
constexpr uint32_t kWarps = kFT / 32;

template <class T>
__device__ __forceinline__ T warp_sum(T v) {
#pragma unroll
  for (uint32_t d = 16; d >= 1; d >>= 1) v += __shfl_xor_sync(0xffffffffu, v, d);
  return v;
}

// --- grid-wide exclusive scan of get(i), i < n -> put(i, prefix); returns the total on every thread.
// Two grid syncs: block sums, then (after every CTA read them) the next user may reuse bsum.
template <class T, class F, class Put>
__device__ T grid_scan(F get, Put put, uint32_t n, T* bsum, cg::grid_group& grid) {
  __shared__ T sh[kWarps + 1];
  const uint32_t lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const uint32_t per = ((n + gridDim.x - 1) / gridDim.x + kFT - 1) / kFT * kFT;
  const uint32_t b0 = min(n, blockIdx.x * per), b1 = min(n, b0 + per);
  T s = 0;
  for (uint32_t i = b0 + threadIdx.x; i < b1; i += kFT) s += get(i);
  s = warp_sum(s);
  if (lane == 0) sh[warp] = s;
  __syncthreads();
  if (threadIdx.x == 0) {
    T t = 0;
    for (uint32_t w = 0; w < kWarps; ++w) t += sh[w];
    bsum[blockIdx.x] = t;
  }
  __syncthreads();
  grid.sync();
  T off = 0, tot = 0;
  for (uint32_t b = threadIdx.x; b < gridDim.x; b += kFT) {
    const T v = bsum[b];
    tot += v;
    if (b < blockIdx.x) off += v;
  }
  off = warp_sum(off);
  tot = warp_sum(tot);
  __syncthreads();
  if (lane == 0) sh[warp] = off;
  __syncthreads();
  if (threadIdx.x == 0) {
    T a = 0;
    for (uint32_t w = 0; w < kWarps; ++w) a += sh[w];
    sh[kWarps] = a;
  }
  __syncthreads();
  off = sh[kWarps];
  __syncthreads();
  if (lane == 0) sh[warp] = tot;
  __syncthreads();
  if (threadIdx.x == 0) {
    T a = 0;
    for (uint32_t w = 0; w < kWarps; ++w) a += sh[w];
    sh[kWarps] = a;
  }
  __syncthreads();
  tot = sh[kWarps];
  __syncthreads();
  // block-level scan of the CTA's range in chunks of kFT, offset by the earlier CTAs' sums
  for (uint32_t base = b0; base < b1; base += kFT) {
    const uint32_t i = base + threadIdx.x;
    const T v = i < b1 ? get(i) : T(0);
    T x = v;
#pragma unroll
    for (uint32_t d = 1; d < 32; d <<= 1) {
      const T y = __shfl_up_sync(0xffffffffu, x, d);
      if (lane >= d) x += y;
    }
    if (lane == 31) sh[warp] = x;
    __syncthreads();
    T woff = 0, ctot = 0;
    for (uint32_t w = 0; w < kWarps; ++w) {
      const T t = sh[w];
      if (w < warp) woff += t;
      ctot += t;
    }
    if (i < b1) put(i, off + woff + x - v);
    off += ctot;
    __syncthreads();
  }
  grid.sync();
  return tot;
}

struct FusedParams {
  const uint32_t* rows;      // bitset rows
  uint64_t pitch;            // words per row
  uint32_t W;                // words in use (ceil(n_tx / 32), multiple of 32 not required)
  uint32_t n1;               // |L_1|
  const uint32_t* sel;       // L_1 entry -> bitset row (nullptr: identity)
  const uint32_t* ior;       // bitset row -> item id
  uint32_t theta, max_k;
  // capacities
  uint32_t cap_cand;         // candidates per generation (M)
  uint32_t cap_words;        // words of an L_k / C_k prefix table (entries x k)
  uint32_t cap_hash;         // power of two
  uint64_t cap_out;          // words of the output arenas (items; supports / counts separately)
  int keep;                  // record every (C_k, counts)
  // candidate buffers (C_k): grouped by (k-1)-prefix
  uint32_t *prefix, *ext_off, *ext, *counts, *pos;
  // levels: L rows (ping-pong), join scratch
  uint32_t *L[2];
  uint32_t *rs, *run_ex, *bound, *cnt, *cand_off, *gidx, *slots[2];
  uint32_t* erun;            // per L_k entry: exclusive run-start count (join_warp's run_ex)
  const uint32_t* c2_counts; // generation 2's counts in pair order, computed before the launch (or nullptr)
  uint32_t *slot, *rowof;    // staging slot of each L_1 entry's row (kNoSlot: unused) and its inverse
  uint32_t* n_used;          // slots assigned
  uint32_t *pslot, *eslot;   // C_k's prefix / extension rows as staging slots
  uint32_t* bsum;            // grid_scan block sums (u32)
  uint64_t* bsum64;          // (u64)
  uint32_t* sink;            // join outputs nobody reads here (the group's left parent, the right parent)
  uint64_t* tstamp;          // GPA_FUSED_TRACE: %globaltimer at every phase boundary (64 x 16)
  uint32_t zsplit;           // word slices per group in the counting phase (>= 1)
  // outputs: per generation k (index k): {M_k, F_k, G_k, freq arena offset (lo, hi), cand arena offset (lo, hi)}
  uint32_t* level_tab;       // 8 words per generation, GPA_MAX_K + 1 generations
  uint32_t *out_items, *out_sup, *cand_items, *cand_counts;
  uint32_t* status;          // [0] bit 1: overflow, [1] generations done
};

__device__ __forceinline__ const uint32_t* row_ptr(const FusedParams& P, uint32_t r) {
  return P.rows + (uint64_t)(P.sel ? P.sel[r] : r) * P.pitch;
}

// ---- the team running a generation: the whole grid (grid.sync, grid-wide scans)
struct GridTeam {
  cg::grid_group& grid;
  __device__ uint32_t tid() const { return blockIdx.x * blockDim.x + threadIdx.x; }
  __device__ uint32_t nthreads() const { return gridDim.x * blockDim.x; }
  __device__ void sync() const { grid.sync(); }
  template <class T, class F, class Put>
  __device__ T scan(F get, Put put, uint32_t n, T* bsum) const { return grid_scan<T>(get, put, n, bsum, grid); }
};
// counts[m] += popcount of the AND of candidate m's rows over a batch of 32-word tiles: work item
// = (tile batch, range of prefix groups); the CTA stages the batch of EVERY L_1 row in shared
// memory (kFusedStageWords words: 64 / |L_1| tiles, or one tile of |L_1| x 32 words), then a warp per group: its structure (prefix rows,
// extensions) loaded once into lanes, per tile the prefix AND from shared memory (lane = word),
// one AND + POPC per extension, warp-reduced (redux.sync), accumulated per extension in the lane
// of that extension; one atomic per (candidate, item).  counts must be zero.
template <class Team>
__device__ void count_phase(const Team& T, const FusedParams& P, uint32_t G, uint32_t km1, uint32_t n_ranges,
                            uint32_t tb, uint32_t nu) {
  extern __shared__ uint32_t s_tile[];   // max(8,192, |L_1| x 32) words (dynamic)
  const uint32_t lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
  const uint32_t n_tiles = (P.W + 31) / 32, n_batches = (n_tiles + tb - 1) / tb;
  const uint32_t gpr = (G + n_ranges - 1) / n_ranges;   // groups per range
  const uint32_t cta = T.tid() / kFT, n_cta = T.nthreads() / kFT;
  for (uint32_t it = cta; it < n_batches * n_ranges; it += n_cta) {
    const uint32_t bt = it % n_batches, r = it / n_batches;   // consecutive CTAs: same range, next batch
    const uint32_t t0 = bt * tb, nt = min(tb, n_tiles - t0);
    __syncthreads();   // the previous item's readers are done with s_tile
    // s_tile[(tile * nu + slot) * 32 + word]: only the rows this generation's candidates use
    for (uint32_t x = wib; x < nt * nu; x += kWarps) {
      const uint32_t tl = x / nu, sl = x % nu;
      const uint32_t row = P.rowof[sl];
      const uint32_t w = 32 * (t0 + tl) + lane;
      s_tile[x * 32 + lane] = w < P.W ? __ldg(P.rows + (uint64_t)(P.sel ? P.sel[row] : row) * P.pitch + w) : 0u;
    }
    __syncthreads();
    const uint32_t g1 = min(G, (r + 1) * gpr);
    for (uint32_t g = r * gpr + wib; g < g1; g += kWarps) {
      const uint32_t e0 = P.ext_off[g], e1 = P.ext_off[g + 1];
      const uint32_t* prg = P.pslot + (uint64_t)g * km1;   // the candidates' rows as staging slots
      const uint32_t my_pre = lane < km1 ? prg[lane] : 0u;  // prefix slots 0..31 in lanes, later ones loaded
      for (uint32_t b0 = e0; b0 < e1; b0 += 32) {
        const uint32_t nb = min(32u, e1 - b0);
        const uint32_t my_ext = lane < nb ? P.eslot[b0 + lane] : 0u;
        uint32_t mine = 0;   // lane j: extension j's count over this item
        for (uint32_t tl = 0; tl < nt; ++tl) {
          const uint32_t* st = s_tile + tl * nu * 32 + lane;
          uint32_t pw = 0xffffffffu;
          for (uint32_t d = 0; d < km1; ++d)
            pw &= st[(d < 32 ? __shfl_sync(0xffffffffu, my_pre, d) : prg[d]) * 32];
          for (uint32_t j = 0; j < nb; ++j) {
            const uint32_t c = __reduce_add_sync(0xffffffffu,
                                                 (uint32_t)__popc(pw & st[__shfl_sync(0xffffffffu, my_ext, j) * 32]));
            mine += lane == j ? c : 0u;
          }
        }
        if (lane < nb && mine) atomicAdd(&P.counts[b0 + lane], mine);
      }
    }
  }
}

__device__ __forceinline__ void stamp(const FusedParams& P, uint32_t k, uint32_t ph) {
  if (P.tstamp && blockIdx.x == 0 && threadIdx.x == 0) {
    uint64_t t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    P.tstamp[(k % 64) * 16 + ph] = t;
  }
}

struct GenState {
  uint32_t k, M, G;
  uint64_t fw, fn, cw, cn;   // output arenas: words / entries so far (frequent, candidates)
  uint32_t done;             // 0: next generation; 1: finished; 2: overflow
  uint32_t hcap_prev;        // slots the previous generation's hash set used (dirty)
  uint32_t n_used;           // rows with a staging slot (the rows of L_{k-1})
};

// One generation by a team: count C_k, threshold into L_k (+ outputs), join + prune into C_{k+1}.
// Every team thread returns the same state.
template <class Team>
__device__ GenState generation(const Team& T, const FusedParams& P, GenState S) {
  const uint32_t tid = T.tid(), n_threads = T.nthreads();
  const uint32_t gw = tid >> 5, n_warps = n_threads >> 5;
  const uint32_t k = S.k, km1 = k - 1, M = S.M, G = S.G;
  // ---- count C_k: (tile batch, group range) items, about two per CTA
  const uint32_t n_tiles = (P.W + 31) / 32;
  const uint32_t nu = S.n_used;   // rows C_k uses (slots assigned while L_{k-1} was scattered)
  const uint32_t tb = max(1u, kFusedStageWords / (32 * max(nu, 1u)));   // tiles per batch (>= kFusedStageWords staged words)
  const uint32_t n_batches = (n_tiles + tb - 1) / tb;
  const uint32_t n_cta = n_threads / kFT;
  const uint32_t n_ranges = max(1u, min(G, (2 * n_cta + n_batches - 1) / n_batches));
  stamp(P, k, 0);
  if (!(k == 2 && P.c2_counts)) {   // (generation 2 counted by the tensor-core pair Gram before the launch)
    count_phase(T, P, G, km1, n_ranges, tb, nu);
    T.sync();
  }
  stamp(P, k, 1);
  // ---- threshold, run structure and hash set of L_k in ONE scan over the groups: group g holds
  // nf_g frequent candidates (consecutive in L_k, lexicographic) and is a run of L_k when nf_g > 0
  // (its members share the group's k-1 prefix) -> (L_k offset, run index) = scan of
  // (nf_g << 32 | nf_g > 0)
  const uint32_t theta = P.theta;
  const uint32_t* counts = P.counts;
  const uint32_t* xo = P.ext_off;
  uint32_t *loff = P.pos, *rrun = P.run_ex;   // per group: L_k offset, run index
  uint32_t* nfg = P.cnt;   // scratch: frequent candidates per group (warp per group)
  // row slots are reassigned for the rows L_k uses (the next generation's candidates)
  for (uint32_t i = tid; i < nu; i += n_threads) P.slot[P.rowof[i]] = kNoSlot;
  if (tid == 0) *P.n_used = 0;
  {
    const uint32_t ln = threadIdx.x & 31;
    for (uint32_t g = gw; g < G; g += n_warps) {
      uint32_t c = 0;
      for (uint32_t m = xo[g] + ln; m < xo[g + 1]; m += 32) c += counts[m] >= theta;
      c = __reduce_add_sync(0xffffffffu, c);
      if (ln == 0) nfg[g] = c;
    }
  }
  T.sync();
  const uint64_t FR = T.template scan<uint64_t>(
      [&](uint32_t g) {
        const uint32_t c = nfg[g];
        return ((uint64_t)c << 32) | (c ? 1ull : 0ull);
      },
      [&](uint32_t g, uint64_t v) {
        loff[g] = (uint32_t)(v >> 32);
        rrun[g] = (uint32_t)v;
      },
      G, P.bsum64);
  const uint32_t F = (uint32_t)(FR >> 32), R = (uint32_t)FR;
  stamp(P, k, 2);
  uint32_t* Lk = P.L[k & 1];
  if ((uint64_t)F * k > P.cap_words || S.fw + (uint64_t)F * k > P.cap_out ||
      (P.keep && S.cw + (uint64_t)M * k > P.cap_out)) {
    S.done = 2;
    return S;
  }
  const uint32_t w = k;
  uint32_t* slots = P.slots[k & 1];
  // hash set of L_k sized to it (>= 2|L_k| + 1 slots, >= 1,024): small tables stay in L1 / L2
  uint32_t hcap = 1024;
  while (hcap < 2 * F + 1 && hcap < P.cap_hash) hcap <<= 1;
  const uint32_t mask = hcap - 1;
  // warp per group: its frequent candidates at loff[g] + rank (ballot), their rows, outputs, run
  // starts, run bounds and hash entries; every candidate to the keep arena
  const uint32_t lane = threadIdx.x & 31;
  for (uint32_t g = gw; g < G; g += n_warps) {
    const uint32_t* pr = P.prefix + (uint64_t)g * km1;
    const uint32_t e0 = xo[g], e1 = xo[g + 1];
    uint32_t base = loff[g];
    for (uint32_t m0 = e0; m0 < e1; m0 += 32) {
      const uint32_t m = m0 + lane;
      const bool valid = m < e1;
      const uint32_t c = valid ? counts[m] : 0u;
      const bool freq = valid && c >= theta;
      const uint32_t bal = __ballot_sync(0xffffffffu, freq);
      const uint32_t e = valid ? P.ext[m] : 0u;
      if (freq) {
        const uint32_t rank = __popc(bal & ((1u << lane) - 1u));
        const uint32_t p = base + rank;
        uint32_t* dst = Lk + (uint64_t)p * k;
        uint32_t* od = P.out_items + S.fw + (uint64_t)p * k;
        for (uint32_t d = 0; d < km1; ++d) {
          dst[d] = pr[d];
          od[d] = P.ior[P.sel ? P.sel[pr[d]] : pr[d]];
        }
        dst[km1] = e;
        od[km1] = P.ior[P.sel ? P.sel[e] : e];
        P.out_sup[S.fn + p] = c;
        for (uint32_t d = 0; d < k; ++d) {   // the rows the next generation's candidates can use
          const uint32_t rw = dst[d];
          if (P.slot[rw] == kNoSlot && atomicCAS(&P.slot[rw], kNoSlot, kClaimed) == kNoSlot) {
            const uint32_t sl = atomicAdd(P.n_used, 1u);
            P.rowof[sl] = rw;
            P.slot[rw] = sl;
          }
        }
        const bool start = p == loff[g];
        P.rs[p] = start ? 1u : 0u;
        if (start) P.bound[rrun[g]] = p;
        uint32_t h = (uint32_t)lvl::hash_mix(lvl::raw_hash(dst, w)) & mask;
        while (atomicCAS(&slots[h], lvl::kEmpty, p) != lvl::kEmpty) h = (h + 1) & mask;
      }
      if (P.keep && valid) {
        uint32_t* cd = P.cand_items + S.cw + (uint64_t)m * k;
        for (uint32_t d = 0; d < km1; ++d) cd[d] = P.ior[P.sel ? P.sel[pr[d]] : pr[d]];
        cd[km1] = P.ior[P.sel ? P.sel[e] : e];
        P.cand_counts[S.cn + m] = c;
      }
      base += __popc(bal);
    }
  }
  if (tid == 0) {
    P.bound[R] = F;
    uint32_t* t = P.level_tab + 8 * k;
    t[0] = M;
    t[1] = F;
    t[2] = G;
    P.status[1] = k;
  }
  // the other table (used by generation k - 1) is cleared for generation k + 1
  // the other table (dirty in the region generation k - 1 used) is cleared for generation k + 1
  uint32_t* other = P.slots[(k + 1) & 1];
  for (uint32_t i = tid; i < S.hcap_prev; i += n_threads) other[i] = lvl::kEmpty;
  S.hcap_prev = hcap;
  S.fw += (uint64_t)F * k;
  S.fn += F;
  if (P.keep) {
    S.cw += (uint64_t)M * k;
    S.cn += M;
  }
  if (F < 2 || k == P.max_k) {
    S.done = 1;
    return S;
  }
  T.sync();
  stamp(P, k, 3);
  // per-entry exclusive run index for join_warp (run of entry p = #run starts <= p, minus 1):
  // from the bounds -- entry p is in run r with bound[r] <= p < bound[r + 1]
  uint32_t* rexp = P.erun;
  for (uint32_t r = gw; r < R; r += n_warps)
    for (uint32_t p = P.bound[r] + lane; p < P.bound[r + 1]; p += 32) rexp[p] = r + 1 - P.rs[p];
  T.sync();
  stamp(P, k, 5);
  for (uint32_t x = gw; x < F; x += n_warps)
    lvl::join_warp<false>(x, Lk, w, P.rs, rexp, P.bound, slots, mask, P.cnt, nullptr, nullptr, nullptr, nullptr,
                          nullptr, nullptr, nullptr);
  T.sync();
  stamp(P, k, 6);
  // survivors and non-empty groups in ONE scan: (count << 32) | (count != 0)
  const uint32_t* cntp = P.cnt;
  uint32_t *cop = P.cand_off, *gip = P.gidx;
  const uint64_t MG = T.template scan<uint64_t>(
      [&](uint32_t x) { return ((uint64_t)cntp[x] << 32) | (cntp[x] ? 1ull : 0ull); },
      [&](uint32_t i, uint64_t v) {
        cop[i] = (uint32_t)(v >> 32);
        gip[i] = (uint32_t)v;
      },
      F, P.bsum64);
  T.sync();
  stamp(P, k, 7);
  const uint32_t M2 = (uint32_t)(MG >> 32), G2 = (uint32_t)MG;
  if (M2 > P.cap_cand || (uint64_t)G2 * w > P.cap_words) {
    S.done = 2;
    return S;
  }
  for (uint32_t x = gw; x < F; x += n_warps)
    lvl::join_warp<true>(x, Lk, w, P.rs, P.erun, P.bound, slots, mask, P.cnt, P.cand_off, P.gidx, P.prefix,
                         P.ext_off, P.ext, P.sink, P.sink + P.cap_cand);   // parents: unused here
  if (tid == 0) P.ext_off[G2] = M2;
  for (uint32_t i = tid; i < M2; i += n_threads) P.counts[i] = 0;
  T.sync();
  // C_{k+1}'s rows as staging slots (assigned while L_k was scattered) for the counting phase
  for (uint32_t i = tid; i < M2; i += n_threads) P.eslot[i] = P.slot[P.ext[i]];
  for (uint32_t i = tid; i < G2 * w; i += n_threads) P.pslot[i] = P.slot[P.prefix[i]];
  S.k = k + 1;
  S.M = M2;
  S.G = G2;
  S.n_used = *reinterpret_cast<volatile uint32_t*>(P.n_used);   // complete: phase C was followed by grid syncs
  S.done = M2 ? 0 : 1;
  return S;
}


__global__ void __launch_bounds__(kFT, 1) mine_fused_kernel(FusedParams P) {
  cg::grid_group grid = cg::this_grid();
  const uint32_t tid = blockIdx.x * blockDim.x + threadIdx.x, n_threads = gridDim.x * blockDim.x;
  // ---- C_2 = every pair of L_1 entries, grouped by the first: group a = {a} x (a, n1)
  const uint32_t n1 = P.n1;
  GenState S{2, n1 > 1 ? n1 * (n1 - 1) / 2 : 0, n1 > 1 ? n1 - 1 : 0, 0, 0, 0, 0, 0, 0, n1};
  for (uint32_t r = tid; r < n1; r += n_threads) {   // generation 2: every row, slot = row
    P.slot[r] = r;
    P.rowof[r] = r;
  }
  for (uint32_t a = tid; a < S.G; a += n_threads) {
    P.pslot[a] = a;
    const uint32_t off = a * n1 - a * (a + 1) / 2;
    for (uint32_t b = a + 1; b < n1; ++b) P.eslot[off + (b - a - 1)] = b;
  }
  for (uint32_t a = tid; a < S.G; a += n_threads) {
    P.prefix[a] = a;
    const uint32_t off = a * n1 - a * (a + 1) / 2;   // pair_index(a, a + 1, n1)
    P.ext_off[a] = off;
    for (uint32_t b = a + 1; b < n1; ++b) P.ext[off + (b - a - 1)] = b;
  }
  if (tid == 0) P.ext_off[S.G] = S.M;
  for (uint32_t i = tid; i < S.M; i += n_threads) P.counts[i] = P.c2_counts ? P.c2_counts[i] : 0u;
  for (uint32_t i = tid; i < P.cap_hash; i += n_threads) P.slots[0][i] = P.slots[1][i] = lvl::kEmpty;
  grid.sync();
  GridTeam GT{grid};
  while (S.k <= P.max_k && S.M > 0 && S.done == 0) {
    const uint32_t kk = S.k;
    S = generation(GT, P, S);
    grid.sync();
    stamp(P, kk, 8);
  }
  if (S.done == 2 && tid == 0) P.status[0] |= 1u;
}

}  // namespace
}  // namespace gpa

namespace gpa {
namespace {

// per-thread, per-device persistent workspace of the fused loop (grow-only; sized once)
struct FusedWork {
  PBuf<uint32_t> prefix, ext_off, ext, counts, pos, L0, L1, rs, run_ex, bound, cnt, cand_off, gidx, s0, s1, bsum, sink;
  PBuf<uint64_t> bsum64;
  PBuf<uint32_t> erun, slot, rowof, n_used, pslot, eslot;
  PBuf<uint32_t> level_tab, status, out_items, out_sup, cand_items, cand_counts;
  int grid = 0;
};
FusedWork& fused_work(int device) {
  thread_local std::map<int, FusedWork> w;
  return w[device];
}

constexpr uint32_t kCapCand = 1u << 20;     // candidates of one generation
constexpr uint32_t kCapWords = 1u << 24;    // words of an L_k / prefix table
constexpr uint32_t kCapHash = 1u << 21;     // >= 2 x kCapCand slots
constexpr uint64_t kCapOut = 1ull << 25;    // words of each output arena

}  // namespace

bool fused_eligible(uint32_t n1, uint64_t pitch_words) {
  return n1 >= 1 && n1 <= kFusedMaxRows && (uint64_t)n1 * pitch_words * 4 <= kFusedMaxBitsetBytes;
}

bool mine_fused(const uint32_t* rows, uint64_t pitch_words, uint64_t n_tx, uint32_t n1, const uint32_t* d_sel,
                const uint32_t* d_ior, uint32_t theta, uint32_t max_k, bool keep, int n_sms, cudaStream_t s,
                FusedOut& out, const uint32_t* c2_counts) {
  int device = 0;
  GPA_CUDA(cudaGetDevice(&device));
  FusedWork& W = fused_work(device);
  const size_t dsmem = (size_t)std::max<uint32_t>(kFusedStageWords, 32u * n1) * 4;
  ensure_smem_attr(reinterpret_cast<const void*>(mine_fused_kernel), (int)(kFusedMaxRows * 32 * 4));
  if (!W.grid) {
    int per_sm = 0;
    GPA_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, mine_fused_kernel, kFT, kFusedMaxRows * 32 * 4));
    GPA_REQUIRE(per_sm > 0, GPA_ERR_CUDA, "mine_fused: kernel does not fit an SM");
    W.grid = per_sm * n_sms;   // one CTA per SM at the largest staging size: valid for every launch
  }
  FusedParams P{};
  P.rows = rows;
  P.pitch = pitch_words;
  P.W = (uint32_t)((n_tx + 31) / 32);
  P.n1 = n1;
  P.sel = d_sel;
  P.ior = d_ior;
  P.theta = theta;
  P.max_k = std::min<uint32_t>(max_k, GPA_MAX_K);
  P.cap_cand = kCapCand;
  // GPA_FUSED_TEST_CAP=n: pretend a generation holds at most n candidates (tests drive the overflow
  // fallback to the multi-kernel path with it)
  if (const char* e = getenv("GPA_FUSED_TEST_CAP")) P.cap_cand = std::min<uint32_t>(kCapCand, (uint32_t)atoi(e));
  P.cap_words = kCapWords;
  P.cap_hash = kCapHash;
  P.cap_out = kCapOut;
  P.keep = keep ? 1 : 0;
  P.prefix = W.prefix.ensure(kCapWords);
  P.ext_off = W.ext_off.ensure(kCapCand + 1);
  P.ext = W.ext.ensure(kCapCand);
  P.counts = W.counts.ensure(kCapCand);
  P.pos = W.pos.ensure(kCapCand);
  P.L[0] = W.L0.ensure(kCapWords);
  P.L[1] = W.L1.ensure(kCapWords);
  P.rs = W.rs.ensure(kCapCand);
  P.run_ex = W.run_ex.ensure(kCapCand);
  P.bound = W.bound.ensure(kCapCand + 1);
  P.cnt = W.cnt.ensure(kCapCand);
  P.cand_off = W.cand_off.ensure(kCapCand);
  P.gidx = W.gidx.ensure(kCapCand);
  P.slots[0] = W.s0.ensure(kCapHash);
  P.slots[1] = W.s1.ensure(kCapHash);
  P.bsum = W.bsum.ensure((size_t)W.grid);
  P.bsum64 = W.bsum64.ensure((size_t)W.grid);
  P.sink = W.sink.ensure(2 * (size_t)kCapCand);
  P.erun = W.erun.ensure(kCapCand);
  P.c2_counts = c2_counts;
  P.slot = W.slot.ensure(kFusedMaxRows);
  P.rowof = W.rowof.ensure(kFusedMaxRows);
  P.n_used = W.n_used.ensure(4);
  P.pslot = W.pslot.ensure(kCapWords);
  P.eslot = W.eslot.ensure(kCapCand);

  static thread_local PBuf<uint64_t> tsb;
  const bool trace = getenv("GPA_FUSED_TRACE") != nullptr;
  P.tstamp = trace ? tsb.ensure(64 * 16) : nullptr;
  if (trace) GPA_CUDA(cudaMemsetAsync(P.tstamp, 0, 64 * 16 * 8, s));
  P.level_tab = W.level_tab.ensure(8 * (GPA_MAX_K + 2));
  P.status = P.level_tab;   // words 0..3 of the table (generation rows start at 8 k, k >= 2)
  P.out_items = W.out_items.ensure(kCapOut);
  P.out_sup = W.out_sup.ensure(kCapOut);
  if (keep) {
    P.cand_items = W.cand_items.ensure(kCapOut);
    P.cand_counts = W.cand_counts.ensure(kCapOut);
  }
  GPA_CUDA(cudaMemsetAsync(P.level_tab, 0, 8 * (GPA_MAX_K + 2) * 4, s));
  void* args[] = {&P};
  GPA_CUDA(cudaLaunchCooperativeKernel(reinterpret_cast<const void*>(mine_fused_kernel), W.grid, kFT, args, dsmem, s));
  note_launch();
  // sizes: status + per-generation (M, F, G)
  thread_local struct HostTab {   // page-locked: one D2H of the status words and the table
    uint32_t* p = nullptr;
    HostTab() { GPA_CUDA(cudaHostAlloc(reinterpret_cast<void**>(&p), 8 * (GPA_MAX_K + 2) * 4, cudaHostAllocDefault)); }
    ~HostTab() { if (p) cudaFreeHost(p); }
  } htab;
  const uint32_t* tab = htab.p;
  const uint32_t* st = htab.p;
  GPA_CUDA(cudaMemcpyAsync(htab.p, P.level_tab, 8 * (GPA_MAX_K + 2) * 4, cudaMemcpyDeviceToHost, s));
  stream_wait(s);
  if (trace) {
    std::vector<uint64_t> ts(64 * 16);
    GPA_CUDA(cudaMemcpy(ts.data(), P.tstamp, ts.size() * 8, cudaMemcpyDeviceToHost));
    for (uint32_t k = 2; k <= st[1]; ++k) {
      fprintf(stderr, "[gpa] fused k=%u M=%u:", k, tab[8 * k]);
      for (int ph = 1; ph <= 8; ++ph)
        if (ts[k * 16 + ph] && ts[k * 16 + ph - 1]) fprintf(stderr, " %d:%.1fus", ph, (ts[k * 16 + ph] - ts[k * 16 + ph - 1]) * 1e-3);
      fprintf(stderr, "\n");
    }
  }
  if (st[0] & 1u) return false;   // a capacity was exceeded: the caller runs the multi-kernel path
  out.levels.clear();
  uint64_t fw = 0, fn = 0, cw = 0, cn = 0;
  for (uint32_t k = 2; k <= st[1]; ++k) {
    FusedOut::Level lv;
    lv.k = k;
    lv.M = tab[8 * k];
    lv.F = tab[8 * k + 1];
    lv.G = tab[8 * k + 2];
    lv.freq_word = fw;
    lv.freq_entry = fn;
    lv.cand_word = cw;
    lv.cand_entry = cn;
    fw += (uint64_t)lv.F * k;
    fn += lv.F;
    if (keep) {
      cw += (uint64_t)lv.M * k;
      cn += lv.M;
    }
    out.levels.push_back(lv);
  }
  out.items = out.sup = nullptr;
  if (fw) {
    size_t bytes = (fw + fn) * 4;
    auto* blk = static_cast<uint32_t*>(out.pinned_alloc(bytes));
    out.items = blk;
    out.sup = blk + fw;
    GPA_CUDA(cudaMemcpyAsync(blk, P.out_items, fw * 4, cudaMemcpyDeviceToHost, s));
    GPA_CUDA(cudaMemcpyAsync(blk + fw, P.out_sup, fn * 4, cudaMemcpyDeviceToHost, s));
  }
  out.cand_items.resize(cw);
  out.cand_counts.resize(cn);
  if (cw) GPA_CUDA(cudaMemcpyAsync(out.cand_items.data(), P.cand_items, cw * 4, cudaMemcpyDeviceToHost, s));
  if (cn) GPA_CUDA(cudaMemcpyAsync(out.cand_counts.data(), P.cand_counts, cn * 4, cudaMemcpyDeviceToHost, s));
  stream_wait(s);
  return true;
}

}  // namespace gpa
