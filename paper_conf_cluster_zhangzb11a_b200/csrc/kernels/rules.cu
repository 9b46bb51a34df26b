// Association rules from the frequent itemsets (sm_100a) -- SURVEY.md §8(f) f4, the downstream
// consumer of F that motivates frequent itemset mining in the paper (PAPER.md P4@338-720: "people
// who buy vegetables often also buy salad dressing").  The paper does not define rules; the
// reading (Q19) is Agrawal & Srikant's (ref [2], P28@1007): for a frequent X with
// |X| >= 2 and a non-empty proper subset A of X, the rule A => X \ A holds when
//
//     conf = supp(X) / supp(A) >= minconf = num / den      (exact: supp(X) * den >= num * supp(A)).
//
// A is frequent (downward closure), so supp(A) is in F: a device hash set over F (polynomial hash
// of the sorted items, as in the join's prune) answers it.  One warp per X: lanes walk the subset
// masks 1 .. 2^k - 2 (bit i = X's i-th item in the antecedent), 32 at a time; pass 1 counts the
// rules of every X, an exclusive scan places them, pass 2 writes them in (X, mask) order.
#include <cstdint>
#include <cstdio>
#include <functional>
#include <vector>

#include "../common.h"
#include "../kernels.h"

namespace gpa {
namespace {

constexpr int kT = 256;
constexpr uint32_t kRulesMaxK = GPA_RULES_MAX_K;
constexpr uint32_t kEmpty = 0xffffffffu;
constexpr uint64_t kP = 0x9E3779B97F4A7C15ull | 1ull;

__device__ __forceinline__ uint64_t mix(uint64_t h) {
  h ^= h >> 33;
  h *= 0xFF51AFD7ED558CCDull;
  h ^= h >> 33;
  h *= 0xC4CEB9FE1A85EC53ull;
  h ^= h >> 33;
  return h;
}

// F on the device: itemset i (global index, canonical order) has k = len and items at
// items + item_off[i], sorted ascending; sup[i] its support.
struct FSet {
  const uint32_t* items;
  const uint64_t* item_off;
  const uint32_t* len;
  const uint32_t* sup;
};

__device__ __forceinline__ uint64_t key_hash(const uint32_t* x, uint32_t k) {
  uint64_t h = k, p = kP;
  for (uint32_t i = 0; i < k; ++i) {
    h += (uint64_t)(x[i] + 1) * p;
    p *= kP;
  }
  return mix(h);
}

__global__ void rules_hash_kernel(FSet F, uint32_t n, uint32_t* slots, uint32_t mask) {
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) {
    uint32_t h = (uint32_t)key_hash(F.items + F.item_off[i], F.len[i]) & mask;
    while (atomicCAS(&slots[h], kEmpty, i) != kEmpty) h = (h + 1) & mask;
  }
}

// support of the itemset a[0..k) (must be in F: downward closure), 0 if absent (cannot happen
// for a valid F; counted as "no rule")
__device__ uint32_t lookup(const FSet& F, const uint32_t* slots, uint32_t mask, const uint32_t* a, uint32_t k) {
  uint32_t h = (uint32_t)key_hash(a, k) & mask;
  for (;;) {
    const uint32_t i = slots[h];
    if (i == kEmpty) return 0;
    if (F.len[i] == k) {
      const uint32_t* y = F.items + F.item_off[i];
      bool eq = true;
      for (uint32_t q = 0; q < k && eq; ++q) eq = y[q] == a[q];
      if (eq) return F.sup[i];
    }
    h = (h + 1) & mask;
  }
}

// warp per X (global index x0 + w); EMIT = false: rule count per X; true: write the rules at off[x]
template <bool EMIT>
__global__ void __launch_bounds__(kT) rules_kernel(FSet F, uint32_t x0, uint32_t n, const uint32_t* __restrict__ slots,
                                                   uint32_t hmask, uint64_t num, uint64_t den,
                                                   uint32_t* __restrict__ cnt, const uint64_t* __restrict__ off,
                                                   uint32_t* __restrict__ out_x, uint32_t* __restrict__ out_mask,
                                                   uint32_t* __restrict__ out_supa) {
  const uint32_t lane = threadIdx.x & 31;
  const uint32_t warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5, n_warps = (gridDim.x * blockDim.x) >> 5;
  for (uint32_t w = warp; w < n; w += n_warps) {
    const uint32_t x = x0 + w;
    const uint32_t k = F.len[x];
    if (k < 2 || k > kRulesMaxK) {  // (k > kRulesMaxK is rejected on the host)
      if (!EMIT && lane == 0) cnt[w] = 0;
      continue;
    }
    uint32_t X[kRulesMaxK];
    const uint32_t* xs = F.items + F.item_off[x];
    for (uint32_t q = 0; q < k; ++q) X[q] = xs[q];
    const uint64_t sx = F.sup[x];
    const uint32_t last = (1u << k) - 2;  // masks 1 .. 2^k - 2
    uint64_t here = EMIT ? off[w] : 0;
    uint32_t total = 0;
    for (uint32_t m0 = 1; m0 <= last; m0 += 32) {
      const uint32_t m = m0 + lane;
      bool ok = false;
      uint32_t sa = 0;
      if (m <= last) {
        uint32_t A[kRulesMaxK], ka = 0;
        for (uint32_t q = 0; q < k; ++q)
          if (m >> q & 1u) A[ka++] = X[q];
        sa = lookup(F, slots, hmask, A, ka);
        ok = sa != 0 && sx * den >= num * (uint64_t)sa;
      }
      const uint32_t b = __ballot_sync(0xffffffffu, ok);
      if (EMIT && ok) {
        const uint64_t at = here + __popc(b & ((1u << lane) - 1u));
        out_x[at] = x;
        out_mask[at] = m;
        out_supa[at] = sa;
      }
      here += __popc(b);
      total += __popc(b);
    }
    if (!EMIT && lane == 0) cnt[w] = total;
  }
}

unsigned grid_for(uint64_t n, int n_sms) {
  uint64_t g = (n + kT - 1) / kT;
  const uint64_t cap = (uint64_t)n_sms * 16;
  return (unsigned)(g < 1 ? 1 : (g > cap ? cap : g));
}

}  // namespace

uint64_t device_rules(const uint32_t* items, const uint64_t* item_off, const uint32_t* len, const uint32_t* sup,
                      uint32_t n, uint32_t x0, uint64_t num, uint64_t den, int n_sms, cudaStream_t s,
                      const std::function<uint32_t*(uint64_t)>& host_alloc) {
  if (n == 0 || x0 >= n) return 0;
  const double t0 = wall_ms();
  const FSet F{items, item_off, len, sup};
  uint32_t cap = 16;
  while (cap < 2 * n + 1) cap <<= 1;
  DBuf<uint32_t> slots, cnt;
  DBuf<uint64_t> off;
  slots.alloc(cap, s);
  GPA_CUDA(cudaMemsetAsync(slots.p, 0xff, (size_t)cap * 4, s));
  { rules_hash_kernel<<<grid_for(n, n_sms), kT, 0, s>>>(F, n, slots.p, cap - 1); note_launch(); }
  const uint32_t nx = n - x0;  // X = the itemsets of size >= 2 (a suffix of the canonical order)
  cnt.alloc(nx, s);
  const unsigned grid = grid_for(32ull * nx, n_sms);
  { rules_kernel<false><<<grid, kT, 0, s>>>(F, x0, nx, slots.p, cap - 1, num, den, cnt.p, nullptr, nullptr, nullptr,
                                            nullptr); note_launch(); }
  // u64 offsets: the rule count may exceed 2^32 in principle
  std::vector<uint32_t> hc(nx);
  GPA_CUDA(cudaMemcpyAsync(hc.data(), cnt.p, (size_t)nx * 4, cudaMemcpyDeviceToHost, s));
  GPA_CUDA(cudaStreamSynchronize(s));
  const double t1 = wall_ms();
  std::vector<uint64_t> ho(nx);
  uint64_t tot = 0;
  for (uint32_t i = 0; i < nx; ++i) {
    ho[i] = tot;
    tot += hc[i];
  }
  GPA_REQUIRE(tot < (1ull << 32), GPA_ERR_RANGE, "more than 2^32 rules");
  if (tot == 0) return 0;
  uint32_t* h = host_alloc(tot);   // 3 x tot words: X index, mask, supp(A)
  const double t2 = wall_ms();
  off.alloc(nx, s);
  GPA_CUDA(cudaMemcpyAsync(off.p, ho.data(), (size_t)nx * 8, cudaMemcpyHostToDevice, s));
  DBuf<uint32_t> ox, om, os;
  ox.alloc(tot, s);
  om.alloc(tot, s);
  os.alloc(tot, s);
  { rules_kernel<true><<<grid, kT, 0, s>>>(F, x0, nx, slots.p, cap - 1, num, den, nullptr, off.p, ox.p, om.p, os.p);
    note_launch(); }
  GPA_CUDA(cudaGetLastError());
  GPA_CUDA(cudaMemcpyAsync(h, ox.p, tot * 4, cudaMemcpyDeviceToHost, s));
  GPA_CUDA(cudaMemcpyAsync(h + tot, om.p, tot * 4, cudaMemcpyDeviceToHost, s));
  GPA_CUDA(cudaMemcpyAsync(h + 2 * tot, os.p, tot * 4, cudaMemcpyDeviceToHost, s));
  GPA_CUDA(cudaStreamSynchronize(s));
  if (trace_enabled())
    fprintf(stderr, "[gpa] rules: %u itemsets, %llu rules: hash + count pass %.2f ms, scan + alloc %.2f ms, emit + D2H "
            "%.2f ms\n", n, (unsigned long long)tot, t1 - t0, t2 - t1, wall_ms() - t2);
  return tot;
}

}  // namespace gpa
