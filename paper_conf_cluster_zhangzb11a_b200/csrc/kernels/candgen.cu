// Device-side level transition (sm_100a): threshold + compaction of a generation's counts into
// L_k, and join + prune candidate generation of C_{k+1} from L_k -- so that between two counting
// launches only a few integers (|L_k|, |C_{k+1}|, #groups) cross PCIe.
//
//   L_k = { c in C_k : count(c) >= min_count }   (P13@474; ">=" per DESIGN.md Q1), lexicographic;
//   C_{k+1} = join of L_k members sharing their first k-1 items (trie siblings, P13@1006-1270,
//             Fig. 4 P18@863) + prune: every k-subset must be in L_k (P13@178; Q7),
//             emitted grouped by k-prefix (group prefix = the left parent), lexicographic.
// The same definitions as the host implementation in runtime/candgen.cpp, written for the GPU:
// flags + exclusive scans (CUB) + scatters; prune probes are binary searches in the sorted L_k.
#include <cstdint>
#include <cub/device/device_scan.cuh>

#include "../common.h"
#include "../kernels.h"

namespace gpa {
namespace {

constexpr int kThreads = 256;

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

__global__ void hash_build_kernel(const uint32_t* __restrict__ L, uint32_t n, uint32_t w, uint32_t* slots,
                                  uint32_t mask) {
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) {
    uint32_t h = (uint32_t)hash_mix(raw_hash(L + (uint64_t)i * w, w)) & mask;
    while (atomicCAS(&slots[h], kEmpty, i) != kEmpty) h = (h + 1) & mask;
  }
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

__global__ void flag_ge_kernel(const uint32_t* __restrict__ counts, uint32_t M, uint32_t theta, uint32_t* flags) {
  for (uint32_t m = blockIdx.x * blockDim.x + threadIdx.x; m < M; m += gridDim.x * blockDim.x)
    flags[m] = counts[m] >= theta;
}

// k = 2: candidate m is the pair (a, b) of pair_index order over n rows
__global__ void scatter_pairs_kernel(const uint32_t* __restrict__ counts, const uint32_t* __restrict__ flags,
                                     const uint32_t* __restrict__ pos, uint32_t M, uint32_t n,
                                     const uint32_t* __restrict__ sel, uint32_t* L,
                                     uint32_t* sup, uint32_t* par_a, uint32_t* par_b) {
  for (uint32_t m = blockIdx.x * blockDim.x + threadIdx.x; m < M; m += gridDim.x * blockDim.x) {
    if (!flags[m]) continue;
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
    const uint32_t p = pos[m];
    L[2ull * p] = a;
    L[2ull * p + 1] = b;
    sup[p] = counts[m];
    par_a[p] = a;
    par_b[p] = b;
  }
}

// k >= 3: candidate m = prefix[g] ++ ext[m] with g the group holding m
__global__ void scatter_grouped_kernel(const uint32_t* __restrict__ counts, const uint32_t* __restrict__ flags,
                                       const uint32_t* __restrict__ pos, uint32_t M,
                                       const uint32_t* __restrict__ prefix, const uint32_t* __restrict__ ext_off,
                                       const uint32_t* __restrict__ ext, uint32_t G, uint32_t km1,
                                       const uint32_t* __restrict__ gpar, const uint32_t* __restrict__ eidx,
                                       uint32_t* L, uint32_t* sup, uint32_t* par_a, uint32_t* par_b) {
  for (uint32_t m = blockIdx.x * blockDim.x + threadIdx.x; m < M; m += gridDim.x * blockDim.x) {
    if (!flags[m]) continue;
    uint32_t lo = 0, hi = G;  // g = last group with ext_off[g] <= m
    while (lo + 1 < hi) {
      const uint32_t mid = (lo + hi) >> 1;
      if (ext_off[mid] <= m) lo = mid; else hi = mid;
    }
    const uint32_t p = pos[m];
    uint32_t* dst = L + (uint64_t)p * (km1 + 1);
    for (uint32_t d = 0; d < km1; ++d) dst[d] = prefix[(uint64_t)lo * km1 + d];
    dst[km1] = ext[m];
    sup[p] = counts[m];
    if (gpar) {
      par_a[p] = gpar[lo];
      par_b[p] = eidx[m];
    }
  }
}

// run starts: members whose first w-1 items differ from the previous member's
__global__ void run_start_kernel(const uint32_t* __restrict__ L, uint32_t n, uint32_t w, uint32_t* flags) {
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x)
    flags[i] = i == 0 || lex_cmp(L + (uint64_t)(i - 1) * w, L + (uint64_t)i * w, w - 1) != 0;
}

__global__ void run_bound_kernel(const uint32_t* __restrict__ flags, const uint32_t* __restrict__ run_ex,
                                 uint32_t n, uint32_t* bound) {
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x)
    if (flags[i]) bound[run_ex[i]] = i;
}

// join + prune of member x with its later run siblings; EMIT = false counts survivors, EMIT = true
// writes group x (prefix = L[x]) and its extensions at the scanned offsets
// Join + prune of member x with its later run siblings, one WARP per x: lane j tests sibling
// y = x + 1 + j (+32 ...); EMIT = false counts survivors, EMIT = true writes group x (prefix = L[x])
// and its extensions, in sibling order, at the scanned offsets (warp ballot ranks the survivors).
template <bool EMIT>
__global__ void join_kernel(const uint32_t* __restrict__ L, uint32_t n, uint32_t w, const uint32_t* __restrict__ flags,
                            const uint32_t* __restrict__ run_ex, const uint32_t* __restrict__ bound,
                            const uint32_t* __restrict__ slots, uint32_t mask, uint32_t* cnt,
                            const uint32_t* __restrict__ cand_off, const uint32_t* __restrict__ gidx,
                            uint32_t* prefix, uint32_t* ext_off, uint32_t* ext, uint32_t* gpar, uint32_t* eidx) {
  uint32_t probe[GPA_MAX_K];
  uint64_t A[GPA_MAX_K], B[GPA_MAX_K];
  const uint32_t lane = threadIdx.x & 31;
  const uint32_t warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5, n_warps = (gridDim.x * blockDim.x) >> 5;
  for (uint32_t x = warp; x < n; x += n_warps) {
    if (EMIT && cnt[x] == 0) continue;  // warp-uniform
    // run index of x = (#run starts <= x) - 1
    const uint32_t r = run_ex[x] + flags[x] - 1;
    const uint32_t end = bound[r + 1];  // bound[n_runs] = n (sentinel)
    if (!EMIT && end == x + 1) {
      if (lane == 0) cnt[x] = 0;
      continue;
    }
    const uint32_t* px = L + (uint64_t)x * w;
    // subset "px without item d, then b": A[d] = sum_{i<d} (x_i+1) P^i,
    // B[d] = sum_{i>d} (x_i+1) P^(i-1); b lands at position w-1
    uint64_t pw = 1, acc = 0;
    for (uint32_t i = 0; i < w; ++i) {  // B[i] temporarily holds P^i
      A[i] = acc;
      B[i] = pw;
      acc += (uint64_t)(px[i] + 1) * pw;
      pw *= kHashP;
    }
    const uint64_t p_last = B[w - 1];  // P^(w-1)
    uint64_t suf = 0;
    for (uint32_t d = w; d-- > 0;) {
      const uint64_t pprev = d > 0 ? B[d - 1] : 0;
      B[d] = suf;
      suf += (uint64_t)(px[d] + 1) * pprev;  // term of item d at position d-1
    }
    uint32_t here = 0;  // survivors so far (warp-uniform)
    for (uint32_t y0 = x + 1; y0 < end; y0 += 32) {
      const uint32_t y = y0 + lane;
      bool keep = y < end;
      uint32_t b = 0;
      if (keep) {
        b = L[(uint64_t)y * w + w - 1];
        const uint64_t hb = (uint64_t)(b + 1) * p_last;
        // subsets dropping item d of the shared prefix (dropping either of the last two items
        // gives the parents x or y, members of L by construction)
        for (uint32_t d = 0; d + 1 < w && keep; ++d) {
          uint32_t q = 0;
          for (uint32_t i = 0; i < w; ++i)
            if (i != d) probe[q++] = px[i];
          probe[q] = b;
          keep = contains(L, w, slots, mask, probe, A[d] + B[d] + hb);
        }
      }
      const uint32_t ballot = __ballot_sync(0xffffffffu, keep);
      if (EMIT && keep) {
        const uint32_t at = cand_off[x] + here + __popc(ballot & ((1u << lane) - 1u));
        ext[at] = b;
        eidx[at] = y;
      }
      here += __popc(ballot);
    }
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
}

// sizes on the device: tot[0] = sum of an exclusive scan (last scanned + last input)
__global__ void total_kernel(const uint32_t* __restrict__ in, const uint32_t* __restrict__ ex, uint32_t n,
                             uint32_t* tot) {
  if (threadIdx.x == 0 && blockIdx.x == 0) *tot = ex[n - 1] + in[n - 1];
}
// bound[n_runs] = n (sentinel end of the last run)
__global__ void bound_sentinel_kernel(const uint32_t* __restrict__ flags, const uint32_t* __restrict__ run_ex,
                                      uint32_t n, uint32_t* bound) {
  if (threadIdx.x == 0 && blockIdx.x == 0) bound[run_ex[n - 1] + flags[n - 1]] = n;
}
// ext_off[G] = M
__global__ void ext_end_kernel(const uint32_t* __restrict__ sizes, uint32_t* ext_off) {
  if (threadIdx.x == 0 && blockIdx.x == 0) ext_off[sizes[1]] = sizes[0];
}

__global__ void nonzero_kernel(const uint32_t* __restrict__ cnt, uint32_t n, uint32_t* flags) {
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x)
    flags[i] = cnt[i] != 0;
}

__global__ void map_items_kernel(const uint32_t* __restrict__ rows, uint64_t n, const uint32_t* __restrict__ ior,
                                 uint32_t* items) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x)
    items[i] = ior[rows[i]];
}

unsigned grid_for(uint64_t n, int n_sms) {
  uint64_t g = (n + kThreads - 1) / kThreads;
  const uint64_t cap = (uint64_t)n_sms * 16;
  return (unsigned)(g < 1 ? 1 : (g > cap ? cap : g));
}

// exclusive scan of n u32 into out, total written to *tot on the device (no host sync)
void exclusive_scan(const uint32_t* in, uint32_t* out, uint32_t n, uint32_t* tot, DeviceScratch& scratch,
                    cudaStream_t s) {
  size_t bytes = 0;
  GPA_CUDA(cub::DeviceScan::ExclusiveSum(nullptr, bytes, in, out, n, s));
  void* tmp = scratch.get(bytes, s);
  GPA_CUDA(cub::DeviceScan::ExclusiveSum(tmp, bytes, in, out, n, s));
  note_launch(2);  // CUB: init + scan kernels
  if (tot) { total_kernel<<<1, 32, 0, s>>>(in, out, n, tot); note_launch(); }
}

}  // namespace

uint32_t device_threshold(const uint32_t* counts, uint32_t M, uint32_t theta, uint32_t k, uint32_t n_rows,
                          const uint32_t* sel, const uint32_t* prefix, const uint32_t* ext_off, const uint32_t* ext,
                          uint32_t G, const uint32_t* gpar, const uint32_t* eidx,
                          DeviceLevel& out, DeviceScratch& scratch, int n_sms, cudaStream_t s) {
  out.k = k;
  out.n = 0;
  if (M == 0) return 0;
  uint32_t* flags = scratch.u32a(M, s);
  uint32_t* pos = scratch.u32b(M, s);
  { flag_ge_kernel<<<grid_for(M, n_sms), kThreads, 0, s>>>(counts, M, theta, flags); note_launch(); }
  GPA_CUDA(cudaGetLastError());
  uint32_t* sizes = scratch.u32c(4, s);
  exclusive_scan(flags, pos, M, sizes, scratch, s);
  uint32_t F = 0;
  GPA_CUDA(cudaMemcpyAsync(&F, sizes, 4, cudaMemcpyDeviceToHost, s));
  stream_wait(s);
  out.rows.ensure((size_t)std::max<uint32_t>(F, 1) * k, s);
  out.sup.ensure(std::max<uint32_t>(F, 1), s);
  out.par_a.ensure(std::max<uint32_t>(F, 1), s);
  out.par_b.ensure(std::max<uint32_t>(F, 1), s);
  if (F) {
    if (k == 2)
      { scatter_pairs_kernel<<<grid_for(M, n_sms), kThreads, 0, s>>>(counts, flags, pos, M, n_rows, sel, out.rows.p,
                                                                  out.sup.p, out.par_a.p, out.par_b.p); note_launch(); }
    else
      { scatter_grouped_kernel<<<grid_for(M, n_sms), kThreads, 0, s>>>(counts, flags, pos, M, prefix, ext_off, ext, G,
                                                                    k - 1, gpar, eidx, out.rows.p, out.sup.p,
                                                                    out.par_a.p, out.par_b.p); note_launch(); }
    GPA_CUDA(cudaGetLastError());
  }
  out.n = F;
  return F;
}

void device_exclusive_scan(const uint32_t* in, uint32_t* out, uint32_t n, uint32_t* tot, DeviceScratch& scratch,
                           cudaStream_t s) {
  exclusive_scan(in, out, n, tot, scratch, s);
}

void device_map_items(const uint32_t* rows, uint64_t n, const uint32_t* item_of_row, uint32_t* items, int n_sms,
                      cudaStream_t s) {
  if (n == 0) return;
  { map_items_kernel<<<grid_for(n, n_sms), kThreads, 0, s>>>(rows, n, item_of_row, items); note_launch(); }
  GPA_CUDA(cudaGetLastError());
}

// Stage 1: run detection, hash set, survivor counts and their scans; the sizes (M, G) are left on
// the device (sizes[0], sizes[1]) -- no synchronisation.  Returns false when L has < 2 members.
bool device_candgen_begin(const DeviceLevel& L, DeviceBatch& out, DeviceScratch& scratch, int n_sms, cudaStream_t s,
                          const uint32_t** d_sizes) {
  const uint32_t n = L.n, w = L.k;
  out.k = w + 1;
  out.M = out.G = 0;
  if (n < 2) return false;
  uint32_t* flags = scratch.u32a(n, s);
  uint32_t* run_ex = scratch.u32b(n, s);
  uint32_t* cnt = scratch.u32c(n, s);
  uint32_t* bound = scratch.u32d(n + 1, s);
  uint32_t* sizes = scratch.u32h(4, s);  // [0] = M, [1] = G
  { run_start_kernel<<<grid_for(n, n_sms), kThreads, 0, s>>>(L.rows.p, n, w, flags); note_launch(); }
  GPA_CUDA(cudaGetLastError());
  exclusive_scan(flags, run_ex, n, nullptr, scratch, s);
  { run_bound_kernel<<<grid_for(n, n_sms), kThreads, 0, s>>>(flags, run_ex, n, bound); note_launch(); }
  { bound_sentinel_kernel<<<1, 32, 0, s>>>(flags, run_ex, n, bound); note_launch(); }
  // hash set over L for the prune probes
  uint32_t cap = 16;
  while (cap < 2 * n + 1) cap <<= 1;
  uint32_t* slots = scratch.u32i(cap, s);
  GPA_CUDA(cudaMemsetAsync(slots, 0xff, (size_t)cap * 4, s));
  { hash_build_kernel<<<grid_for(n, n_sms), kThreads, 0, s>>>(L.rows.p, n, w, slots, cap - 1); note_launch(); }
  { join_kernel<false><<<grid_for(32ull * n, n_sms), kThreads, 0, s>>>(L.rows.p, n, w, flags, run_ex, bound, slots, cap - 1, cnt,
                                                             nullptr, nullptr, nullptr, nullptr, nullptr, nullptr, nullptr); note_launch(); }
  GPA_CUDA(cudaGetLastError());
  uint32_t* cand_off = scratch.u32e(n, s);
  uint32_t* gflag = scratch.u32f(n, s);
  uint32_t* gidx = scratch.u32g(n, s);
  exclusive_scan(cnt, cand_off, n, sizes, scratch, s);
  { nonzero_kernel<<<grid_for(n, n_sms), kThreads, 0, s>>>(cnt, n, gflag); note_launch(); }
  exclusive_scan(gflag, gidx, n, sizes + 1, scratch, s);
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
  out.prefix.ensure((size_t)G * w, s);
  out.ext_off.ensure(G + 1, s);
  out.ext.ensure(M, s);
  out.gpar.ensure(G, s);
  out.eidx.ensure(M, s);
  if (run != s) {
    GPA_CUDA(cudaEventRecord(ev, s));
    GPA_CUDA(cudaStreamWaitEvent(run, ev, 0));
  }
  uint32_t cap = 16;
  while (cap < 2 * n + 1) cap <<= 1;
  { join_kernel<true><<<grid_for(32ull * n, n_sms), kThreads, 0, run>>>(L.rows.p, n, w, scratch.a.p, scratch.b.p,
        scratch.d.p, scratch.i.p, cap - 1, scratch.c.p, scratch.e.p, scratch.g.p, out.prefix.p, out.ext_off.p,
        out.ext.p, out.gpar.p, out.eidx.p); note_launch(); }
  GPA_CUDA(cudaGetLastError());
  { ext_end_kernel<<<1, 32, 0, run>>>(scratch.h.p, out.ext_off.p); note_launch(); }
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
