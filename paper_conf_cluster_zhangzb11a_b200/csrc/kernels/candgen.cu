// Device-side level transition (sm_100a): threshold + compaction of a generation's counts into
// L_k, and join + prune candidate generation of C_{k+1} from L_k -- so that between two counting
// launches only a few integers (|L_k|, |C_{k+1}|, #groups) cross PCIe.
//
//   L_k = { c in C_k : count(c) >= min_count }   (P13@474; ">=" per DESIGN.md Q1), lexicographic;
//   C_{k+1} = join of L_k members sharing their first k-1 items (trie siblings, P13@1006-1270,
//             Fig. 4 P18@863) + prune: every k-subset must be in L_k (P13@178; Q7),
//             emitted grouped by k-prefix (group prefix = the left parent), lexicographic.
// The same definitions as the host implementation in runtime/candgen.cpp, written for the GPU:
// single-launch scans with fused flags / bounds (scan_dev.cuh) + scatters; prune probes hit a
// device hash set over L_k (level_dev.cuh).
#include <cstdint>

#include "../common.h"
#include "../kernels.h"
#include "level_dev.cuh"
#include "scan_dev.cuh"

namespace gpa {
namespace {
using namespace lvl;

constexpr int kThreads = 128;
constexpr int kRunScanItems = 2;   // run detection compares two rows per member: more CTAs in flight

// n_dev (device-sized levels): the member count lives on the device; n is its host upper bound
__device__ __forceinline__ uint32_t eff_n(uint32_t n, const uint32_t* n_dev) { return n_dev ? min(*n_dev, n) : n; }

// entry p (its w row ids at row) into the hash set of the next join's prune probes -- done by the
// scatter that writes L_k, so the set needs no pass of its own (slots cleared to kEmpty first)
__device__ __forceinline__ void hash_insert(const uint32_t* row, uint32_t w, uint32_t p, uint32_t* slots,
                                            uint32_t mask) {
  uint32_t h = (uint32_t)hash_mix(raw_hash(row, w)) & mask;
  while (atomicCAS(&slots[h], kEmpty, p) != kEmpty) h = (h + 1) & mask;
}

// L_k's positions: pos[m] = #{m' < m : count >= theta}, *count = |L_k| (one launch)
__global__ void __launch_bounds__(sd::kScanThreads, 1) ge_scan_kernel(const uint32_t* __restrict__ counts, uint32_t M,
                                                                      uint32_t theta, uint32_t* __restrict__ pos,
                                                                      uint32_t* count, uint32_t* count2, uint32_t* sflags,
                                                                      uint64_t* agg, uint64_t* inc, uint32_t epoch) {
  sd::scan_tile<uint32_t>(
      M, [&](uint32_t m) { return counts[m] >= theta ? 1u : 0u; }, [&](uint32_t m, uint32_t e, uint32_t) { pos[m] = e; },
      [&](uint32_t t) {
        *count = t;
        if (count2) *count2 = t;   // |L_k| into the next generation's size block as well
      },
      sflags, agg, inc, epoch);
}

// k = 2: candidate m is the pair (a, b) of pair_index order over n rows
// (every scatter also writes the entry's original item ids and support for the result: ior maps a
// bitset row to its item id; items / sup_out may be null)
struct ScatterOut {   // L_k and the side outputs one frequent candidate is scattered into
  uint32_t *L, *sup, *par_a, *par_b;
  const uint32_t* ior;
  uint32_t *items, *sup_out, *slots;
  uint32_t mask;
};

__device__ __forceinline__ void scatter_pair(uint32_t m, uint32_t p, uint32_t c, uint32_t n,
                                             const uint32_t* __restrict__ sel, const ScatterOut& o) {
  uint32_t lo = 0, hi = n - 1;  // a = last row whose first pair index <= m
  while (lo + 1 < hi) {
    const uint32_t mid = (lo + hi) >> 1;
    if (pair_index(mid, mid + 1, n) <= m) lo = mid; else hi = mid;
  }
  uint32_t a = lo, b = (uint32_t)(m - pair_index(a, a + 1, n)) + a + 1;
  if (sel) {   // logical L_1 indices -> bitset rows
    a = sel[a];
    b = sel[b];
  }
  o.L[2ull * p] = a;
  o.L[2ull * p + 1] = b;
  o.sup[p] = c;
  o.par_a[p] = a;
  o.par_b[p] = b;
  if (o.items) {
    o.items[2ull * p] = o.ior[a];
    o.items[2ull * p + 1] = o.ior[b];
    o.sup_out[p] = c;
  }
  if (o.slots) hash_insert(o.L + 2ull * p, 2, p, o.slots, o.mask);
}

// k >= 3: candidate m = prefix[g] ++ ext[m] with g the group holding m
__device__ __forceinline__ void scatter_grouped(uint32_t m, uint32_t p, uint32_t c,
                                                const uint32_t* __restrict__ prefix,
                                                const uint32_t* __restrict__ ext_off, const uint32_t* __restrict__ ext,
                                                uint32_t G, uint32_t km1, const uint32_t* __restrict__ gpar,
                                                const uint32_t* __restrict__ eidx, const ScatterOut& o) {
  uint32_t lo = 0, hi = G;  // g = last group with ext_off[g] <= m
  while (lo + 1 < hi) {
    const uint32_t mid = (lo + hi) >> 1;
    if (ext_off[mid] <= m) lo = mid; else hi = mid;
  }
  uint32_t* dst = o.L + (uint64_t)p * (km1 + 1);
  uint32_t* it = o.items ? o.items + (uint64_t)p * (km1 + 1) : nullptr;
  for (uint32_t d = 0; d < km1; ++d) {
    const uint32_t r = prefix[(uint64_t)lo * km1 + d];
    dst[d] = r;
    if (it) it[d] = o.ior[r];
  }
  dst[km1] = ext[m];
  o.sup[p] = c;
  if (it) {
    it[km1] = o.ior[ext[m]];
    o.sup_out[p] = c;
  }
  if (o.slots) hash_insert(dst, km1 + 1, p, o.slots, o.mask);
  if (gpar) {
    o.par_a[p] = gpar[lo];
    o.par_b[p] = eidx[m];
  }
}

// The threshold in ONE launch: the flag scan of counts >= theta, each frequent candidate scattered
// at its exclusive rank in the scan's output phase (after the tile's look-back: the scatters do not
// delay later tiles), |L_k| from the last tile.  k2: pair order (generation 2), else grouped.
template <bool K2>
__global__ void __launch_bounds__(sd::kScanThreads, 1) ge_scatter_kernel(
    const uint32_t* __restrict__ counts, uint32_t M, uint32_t theta, uint32_t n, const uint32_t* __restrict__ sel,
    const uint32_t* __restrict__ prefix, const uint32_t* __restrict__ ext_off, const uint32_t* __restrict__ ext,
    uint32_t G, uint32_t km1, const uint32_t* __restrict__ gpar, const uint32_t* __restrict__ eidx, ScatterOut o,
    uint32_t* count, uint32_t* count2, uint32_t* sflags, uint64_t* agg, uint64_t* inc, uint32_t epoch) {
  sd::scan_tile<uint32_t, 4>(
      M, [&](uint32_t m) { return counts[m] >= theta ? 1u : 0u; },
      [&](uint32_t m, uint32_t e, uint32_t f) {
        if (!f) return;
        if constexpr (K2) scatter_pair(m, e, counts[m], n, sel, o);
        else scatter_grouped(m, e, counts[m], prefix, ext_off, ext, G, km1, gpar, eidx, o);
      },
      [&](uint32_t t) {
        *count = t;
        if (count2) *count2 = t;
      },
      sflags, agg, inc, epoch);
}

// run starts (members whose first w-1 items differ from the previous member's; zero past the
// device count: the scans run over the host upper bound) in one launch: flags, their exclusive
// scan run_ex, bound[r] = the first member of run r and bound[#runs] = |L| (the sentinel)
__global__ void __launch_bounds__(sd::kScanThreads, 1) run_scan_kernel(const uint32_t* __restrict__ L, uint32_t n,
                                                                       uint32_t w, uint32_t* __restrict__ flags,
                                                                       uint32_t* __restrict__ run_ex,
                                                                       uint32_t* __restrict__ bound,
                                                                       const uint32_t* __restrict__ n_dev,
                                                                       uint32_t* sflags, uint64_t* agg, uint64_t* inc,
                                                                       uint32_t epoch) {
  const uint32_t ne = eff_n(n, n_dev);
  sd::scan_tile<uint32_t, kRunScanItems>(
      n,
      [&](uint32_t i) {
        const uint32_t f = i < ne && (i == 0 || lex_cmp(L + (uint64_t)(i - 1) * w, L + (uint64_t)i * w, w - 1) != 0);
        flags[i] = f;
        return f;
      },
      [&](uint32_t i, uint32_t e, uint32_t f) {
        run_ex[i] = e;
        if (f) bound[e] = i;
      },
      [&](uint32_t runs) { bound[runs] = ne; }, sflags, agg, inc, epoch);
}

// join + prune, one WARP per member x (lvl::join_warp)
template <bool EMIT>
__global__ void join_kernel(const uint32_t* __restrict__ L, uint32_t n, uint32_t w, const uint32_t* __restrict__ flags,
                            const uint32_t* __restrict__ run_ex, const uint32_t* __restrict__ bound,
                            const uint32_t* __restrict__ slots, uint32_t mask, uint32_t* cnt,
                            const uint32_t* __restrict__ cand_off, const uint32_t* __restrict__ gidx,
                            uint32_t* prefix, uint32_t* ext_off, uint32_t* ext, uint32_t* gpar, uint32_t* eidx,
                            const uint32_t* __restrict__ n_dev, const uint32_t* __restrict__ sizes,
                            unsigned long long* surv) {
  const uint32_t warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5, n_warps = (gridDim.x * blockDim.x) >> 5;
  const uint32_t ne = eff_n(n, n_dev);
  if (EMIT && blockIdx.x == 0 && threadIdx.x == 0) ext_off[sizes[1]] = sizes[0];   // ext_off[G] = M
  for (uint32_t x = warp; x < n; x += n_warps) {
    if (x < ne)
      lvl::join_warp<EMIT>(x, L, w, flags, run_ex, bound, slots, mask, cnt, cand_off, gidx, prefix, ext_off, ext,
                           gpar, eidx, surv);
    else if (!EMIT && (threadIdx.x & 31) == 0)
      cnt[x] = 0;   // past the device count: no survivors (the scans run over the upper bound)
  }
}

// L_k's rows -> item ids (n = entries x k words) and, with sup_in, its supports copied to sup_out;
// a device-sized level stops at its count
__global__ void map_items_kernel(const uint32_t* __restrict__ rows, uint64_t n, const uint32_t* __restrict__ ior,
                                 uint32_t* items, const uint32_t* __restrict__ n_dev, uint32_t k,
                                 const uint32_t* __restrict__ sup_in, uint32_t* sup_out) {
  if (n_dev && (uint64_t)*n_dev * k < n) n = (uint64_t)*n_dev * k;
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x) {
    items[i] = ior[rows[i]];
    if (sup_in && i % k == 0) sup_out[i / k] = sup_in[i / k];
  }
}

unsigned grid_for(uint64_t n, int n_sms) {
  uint64_t g = (n + kThreads - 1) / kThreads;
  const uint64_t cap = (uint64_t)n_sms * 16;
  return (unsigned)(g < 1 ? 1 : (g > cap ? cap : g));
}

// exclusive scan of n u32 into out, total written to *tot on the device (no host sync)
void exclusive_scan(const uint32_t* in, uint32_t* out, uint32_t n, uint32_t* tot, DeviceScratch& scratch,
                    cudaStream_t s) {
  scan_excl_u32(in, out, n, tot, scratch.scan, s);   // one launch, total included (scan.cu)
}

void ge_scan(const uint32_t* counts, uint32_t M, uint32_t theta, uint32_t* pos, uint32_t* count, DeviceScratch& scratch,
             cudaStream_t s, uint32_t* count2 = nullptr) {
  const uint32_t tiles = scan_tiles(M);
  const uint32_t ep = scan_epoch(scratch.scan, tiles, s);
  { ge_scan_kernel<<<tiles, sd::kScanThreads, 0, s>>>(counts, M, theta, pos, count, count2, scratch.scan.flags.p,
                                                      scratch.scan.agg.p, scratch.scan.inc.p, ep); note_launch(); }
  GPA_CUDA(cudaGetLastError());
}

}  // namespace

namespace {
void threshold_impl(const uint32_t* counts, uint32_t M, uint32_t theta, uint32_t k, uint32_t n_rows, const uint32_t* sel,
                    const uint32_t* prefix, const uint32_t* ext_off, const uint32_t* ext, uint32_t G,
                    const uint32_t* gpar, const uint32_t* eidx, DeviceLevel& out, DeviceScratch& scratch, int n_sms,
                    cudaStream_t s, uint32_t cap, const uint32_t* ior, uint32_t* items, uint32_t* sup_out,
                    uint32_t* count2) {
  out.count.ensure(1, s);
  out.rows.ensure((size_t)std::max<uint32_t>(cap, 1) * k, s);
  out.sup.ensure(std::max<uint32_t>(cap, 1), s);
  out.par_a.ensure(std::max<uint32_t>(cap, 1), s);
  out.par_b.ensure(std::max<uint32_t>(cap, 1), s);
  // the next join's hash set over L_k (sized for the upper bound cap), filled by the scatter
  uint32_t hcap = 16;
  while (hcap < 2 * cap + 1) hcap <<= 1;
  uint32_t* slots = scratch.u32i(hcap, s);
  scratch.hash_cap = hcap;
  scratch.hash_n = cap;
  GPA_CUDA(cudaMemsetAsync(slots, 0xff, (size_t)hcap * 4, s));
  const ScatterOut o{out.rows.p, out.sup.p, out.par_a.p, out.par_b.p, ior, items, sup_out, slots, hcap - 1};
  {   // scan + scatter in one launch
    const uint32_t tiles = scan_tiles(M, 4);
    const uint32_t ep = scan_epoch(scratch.scan, tiles, s);
    if (k == 2)
      ge_scatter_kernel<true><<<tiles, sd::kScanThreads, 0, s>>>(counts, M, theta, n_rows, sel, nullptr, nullptr,
          nullptr, 0, 1, nullptr, nullptr, o, out.count.p, count2, scratch.scan.flags.p, scratch.scan.agg.p,
          scratch.scan.inc.p, ep);
    else
      ge_scatter_kernel<false><<<tiles, sd::kScanThreads, 0, s>>>(counts, M, theta, n_rows, sel, prefix, ext_off,
          ext, G, k - 1, gpar, eidx, o, out.count.p, count2, scratch.scan.flags.p, scratch.scan.agg.p,
          scratch.scan.inc.p, ep);
    note_launch();
  }
  GPA_CUDA(cudaGetLastError());
}
}  // namespace

uint32_t device_threshold(const uint32_t* counts, uint32_t M, uint32_t theta, uint32_t k, uint32_t n_rows,
                          const uint32_t* sel, const uint32_t* prefix, const uint32_t* ext_off, const uint32_t* ext,
                          uint32_t G, const uint32_t* gpar, const uint32_t* eidx,
                          DeviceLevel& out, DeviceScratch& scratch, int n_sms, cudaStream_t s) {
  out.k = k;
  out.n = 0;
  out.n_dev = nullptr;
  out.n_max = 0;
  if (M == 0) return 0;
  // |L_k| first (one synchronisation), then L_k at its exact size
  uint32_t* pos = scratch.u32b(M, s);
  out.count.ensure(1, s);
  ge_scan(counts, M, theta, pos, out.count.p, scratch, s);
  uint32_t F = 0;
  GPA_CUDA(cudaMemcpyAsync(&F, out.count.p, 4, cudaMemcpyDeviceToHost, s));
  stream_wait(s);
  if (F) threshold_impl(counts, M, theta, k, n_rows, sel, prefix, ext_off, ext, G, gpar, eidx, out, scratch, n_sms, s,
                        F, nullptr, nullptr, nullptr, nullptr);
  out.n = F;
  return F;
}

void device_threshold_async(const uint32_t* counts, uint32_t M, uint32_t theta, uint32_t k, uint32_t n_rows,
                            const uint32_t* sel, const uint32_t* prefix, const uint32_t* ext_off, const uint32_t* ext,
                            uint32_t G, const uint32_t* gpar, const uint32_t* eidx,
                            DeviceLevel& out, DeviceScratch& scratch, int n_sms, cudaStream_t s,
                            const uint32_t* ior, uint32_t* items, uint32_t* sup_out) {
  out.k = k;
  out.n = 0;
  out.n_dev = nullptr;
  out.n_max = 0;
  if (M == 0) return;
  threshold_impl(counts, M, theta, k, n_rows, sel, prefix, ext_off, ext, G, gpar, eidx, out, scratch, n_sms, s, M, ior,
                 items, sup_out, scratch.size_block(s) + 10);
  out.n_dev = out.count.p;   // |L_k| stays on the device until the next generation's synchronisation
  out.n_max = M;
}

void device_exclusive_scan(const uint32_t* in, uint32_t* out, uint32_t n, uint32_t* tot, DeviceScratch& scratch,
                           cudaStream_t s) {
  exclusive_scan(in, out, n, tot, scratch, s);
}

void device_map_items(const uint32_t* rows, uint64_t n, const uint32_t* item_of_row, uint32_t* items, int n_sms,
                      cudaStream_t s, const uint32_t* n_dev, uint32_t k, const uint32_t* sup_in, uint32_t* sup_out) {
  if (n == 0) return;
  { map_items_kernel<<<grid_for(n, n_sms), kThreads, 0, s>>>(rows, n, item_of_row, items, n_dev, k, sup_in, sup_out);
    note_launch(); }
  GPA_CUDA(cudaGetLastError());
}

// Stage 1: run detection, hash set, survivor counts and their scans; the sizes (M, G) are left on
// the device (sizes[0], sizes[1]) -- no synchronisation.  Returns false when L has < 2 members.
bool device_candgen_begin(const DeviceLevel& L, DeviceBatch& out, DeviceScratch& scratch, int n_sms, cudaStream_t s,
                          const uint32_t** d_sizes, const uint32_t* run_flags, const uint32_t* run_ex_in,
                          const uint32_t* run_bound) {
  const uint32_t* n_dev = L.n_dev;
  const uint32_t n = n_dev ? L.n_max : L.n, w = L.k;   // device-sized level: n = the host upper bound
  out.k = w + 1;
  out.M = out.G = 0;
  if (n < 2) return false;
  uint32_t* cnt = scratch.u32c(n, s);
  uint32_t* sizes = scratch.size_block(s);  // [0] = M, [1] = G
  // the hash set over L for the prune probes was filled by the scatter that wrote L (threshold_impl)
  GPA_REQUIRE(scratch.hash_cap >= 2 * n + 1 && scratch.hash_n == n && scratch.i.p, GPA_ERR_STATE,
              "join: no hash set over this level");
  const uint32_t cap = scratch.hash_cap;   // the emitting join (stage 2) probes the same table
  uint32_t* slots = scratch.i.p;
  const uint32_t *flags = run_flags, *run_ex = run_ex_in, *bound = run_bound;
  if (!flags) {
    uint32_t* f = scratch.u32a(n, s);
    uint32_t* e = scratch.u32b(n, s);
    uint32_t* b = scratch.u32d(n + 1, s);
    const uint32_t tiles = scan_tiles(n, kRunScanItems);
    const uint32_t ep = scan_epoch(scratch.scan, tiles, s);
    run_scan_kernel<<<tiles, sd::kScanThreads, 0, s>>>(L.rows.p, n, w, f, e, b, n_dev, scratch.scan.flags.p,
                                                       scratch.scan.agg.p, scratch.scan.inc.p, ep);
    note_launch();
    GPA_CUDA(cudaGetLastError());
    flags = f;
    run_ex = e;
    bound = b;
  }
  scratch.rflags = flags;
  scratch.rex = run_ex;
  scratch.rbound = bound;
  { join_kernel<false><<<grid_for(32ull * n, n_sms), kThreads, 0, s>>>(L.rows.p, n, w, flags, run_ex, bound, slots,
        cap - 1, cnt, nullptr, nullptr, nullptr, nullptr, nullptr, nullptr, nullptr, n_dev, nullptr,
        scratch.surv64(n, s)); note_launch(); }
  GPA_CUDA(cudaGetLastError());
  uint32_t* cand_off = scratch.u32e(n, s);
  uint32_t* gidx = scratch.u32g(n, s);
  // candidate offsets and group indices in one scan: sizes = {M, G}
  scan_excl_split(cnt, cand_off, gidx, n, sizes, scratch.scan, s);
  *d_sizes = sizes;
  return true;
}

// Stage 2 (after the host has read M, G): the output buffers are sized on `s`, the emitting join
// runs on `run` (which waits for `s` through `ev`; run == s for a single stream).
void device_candgen_finish(const DeviceLevel& L, DeviceBatch& out, DeviceScratch& scratch, int n_sms, cudaStream_t s,
                           uint32_t M, uint32_t G, cudaStream_t run, cudaEvent_t ev) {
  const uint32_t n = L.n, w = L.k;
  out.M = out.G = 0;
  if (M == 0) return;
  // run != s with ev == nullptr: the caller already made `run` wait for s at the end of stage 1, and s
  // may hold later work -- the batch is then allocated (stream-ordered) on `run` itself
  const cudaStream_t as = run != s && !ev ? run : s;
  out.prefix.ensure((size_t)G * w, as);
  out.ext_off.ensure(G + 1, as);
  out.ext.ensure(M, as);
  out.gpar.ensure(G, as);
  out.eidx.ensure(M, as);
  if (run != s && ev) {
    GPA_CUDA(cudaEventRecord(ev, s));
    GPA_CUDA(cudaStreamWaitEvent(run, ev, 0));
  }
  const uint32_t cap = scratch.hash_cap;   // the table stage 1 built (sized for its upper bound)
  { join_kernel<true><<<grid_for(32ull * n, n_sms), kThreads, 0, run>>>(L.rows.p, n, w, scratch.rflags, scratch.rex,
        scratch.rbound, scratch.i.p, cap - 1, scratch.c.p, scratch.e.p, scratch.g.p, out.prefix.p, out.ext_off.p,
        out.ext.p, out.gpar.p, out.eidx.p, nullptr, scratch.blk.p, scratch.surv.p); note_launch(); }   // + ext_off[G] = M
  GPA_CUDA(cudaGetLastError());
  out.M = M;
  out.G = G;
}

void device_candgen(const DeviceLevel& L, DeviceBatch& out, DeviceScratch& scratch, int n_sms, cudaStream_t s) {
  const uint32_t* sizes = nullptr;
  if (!device_candgen_begin(L, out, scratch, n_sms, s, &sizes)) return;
  uint32_t MG[2] = {0, 0};
  GPA_CUDA(cudaMemcpyAsync(MG, sizes, 8, cudaMemcpyDeviceToHost, s));
  stream_wait(s);
  device_candgen_finish(L, out, scratch, n_sms, s, MG[0], MG[1], s, nullptr);
}

}  // namespace gpa
