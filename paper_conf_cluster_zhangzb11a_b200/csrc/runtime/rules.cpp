// Association rules from a mining result (gpa_rules_*, Q19): the
// result's frequent itemsets go to the device once, the rules are enumerated there (rules.cu)
// and come back as three arrays owned by the gpa_rules handle.
#include <sys/mman.h>

#include <algorithm>


#include "internal.h"
#include "pool.h"

// Host buffer for the rules (hundreds of MB): anonymous mapping with transparent huge pages, first
// touched in parallel -- fresh 4 KB pages faulted in one by one by the D2H copy ran at ~2 GB/s.
struct HostWords {
  uint32_t* p = nullptr;
  size_t bytes = 0;
  ~HostWords() {
    if (p) munmap(p, bytes);
  }
  uint32_t* alloc(uint64_t words) {
    bytes = std::max<size_t>(words * 4, 4096);
    void* m = mmap(nullptr, bytes, PROT_READ | PROT_WRITE, MAP_PRIVATE | MAP_ANONYMOUS, -1, 0);
    GPA_REQUIRE(m != MAP_FAILED, GPA_ERR_OOM, "host allocation of %zu bytes failed", bytes);
    p = static_cast<uint32_t*>(m);
#ifdef MADV_HUGEPAGE
    madvise(m, bytes, MADV_HUGEPAGE);
#endif
    const size_t T = std::max<size_t>(1, std::min<size_t>(gpa::pool_threads(), bytes >> 24));
    auto* c = static_cast<volatile uint8_t*>(m);
    gpa::parallel_for(T, [&](size_t t) {
      for (size_t o = bytes * t / T; o < bytes * (t + 1) / T; o += 4096) c[o] = 0;
    });
    return p;
  }
};

struct gpa_rules {
  HostWords data;   // 3 x n words: X indices, masks, supports of A
  uint64_t n = 0;
};

extern "C" gpa_status gpa_rules_create(const gpa_result* r, uint64_t conf_num, uint64_t conf_den, gpa_rules** out) {
  return gpa::guard([&] {
    using namespace gpa;
    GPA_REQUIRE(r && out, GPA_ERR_INVALID, "NULL argument");
    GPA_REQUIRE(conf_den > 0, GPA_ERR_INVALID, "conf_den must be > 0");
    GPA_REQUIRE(conf_num < (1ull << 32) && conf_den < (1ull << 32), GPA_ERR_INVALID, "conf_num, conf_den must be < 2^32");
    *out = nullptr;
    // F in canonical order (the indices of gpa_result_get)
    uint64_t n = 0, x0 = 0;
    uint32_t nl = 0;
    GPA_CUDA(cudaGetLastError());
    {
      gpa_status st = gpa_result_n_levels(r, &nl);
      GPA_REQUIRE(st == GPA_OK, st, "%s", gpa_last_error());
    }
    std::vector<uint32_t> items, len, sup;
    std::vector<uint64_t> off;
    for (uint32_t k = 1; k <= nl; ++k) {
      uint64_t nk = 0;
      const uint32_t *it = nullptr, *su = nullptr;
      gpa_status st = gpa_result_frequent(r, k, &nk, &it, &su);
      GPA_REQUIRE(st == GPA_OK, st, "%s", gpa_last_error());
      if (k == 2) x0 = n;
      GPA_REQUIRE(nk == 0 || k <= GPA_RULES_MAX_K, GPA_ERR_RANGE, "itemsets of %u items (rules support <= %u)", k,
                  GPA_RULES_MAX_K);
      for (uint64_t j = 0; j < nk; ++j) {
        off.push_back(items.size());
        items.insert(items.end(), it + j * k, it + (j + 1) * k);
        len.push_back(k);
        sup.push_back(su[j]);
      }
      n += nk;
    }
    if (nl < 2) x0 = n;
    GPA_REQUIRE(n < (1ull << 32), GPA_ERR_RANGE, "too many itemsets");
    auto* R = new gpa_rules();
    struct G {
      gpa_rules* p;
      ~G() { delete p; }
    } g{R};
    if (n > x0) {
      const DeviceInfo di = use_device(-1);
      cudaStream_t s = nullptr;
      GPA_CUDA(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
      struct SG {
        cudaStream_t s;
        ~SG() { cudaStreamSynchronize(s); cudaStreamDestroy(s); }
      } sg{s};
      DBuf<uint32_t> d_items, d_len, d_sup;
      DBuf<uint64_t> d_off;
      d_items.alloc(std::max<size_t>(items.size(), 1), s);
      d_len.alloc(n, s);
      d_sup.alloc(n, s);
      d_off.alloc(n, s);
      GPA_CUDA(cudaMemcpyAsync(d_items.p, items.data(), items.size() * 4, cudaMemcpyHostToDevice, s));
      GPA_CUDA(cudaMemcpyAsync(d_len.p, len.data(), n * 4, cudaMemcpyHostToDevice, s));
      GPA_CUDA(cudaMemcpyAsync(d_sup.p, sup.data(), n * 4, cudaMemcpyHostToDevice, s));
      GPA_CUDA(cudaMemcpyAsync(d_off.p, off.data(), n * 8, cudaMemcpyHostToDevice, s));
      R->n = device_rules(d_items.p, d_off.p, d_len.p, d_sup.p, (uint32_t)n, (uint32_t)x0, conf_num, conf_den,
                          di.n_sms, s, [&](uint64_t m) { return R->data.alloc(3 * m); });
    }
    *out = R;
    g.p = nullptr;
  });
}

extern "C" gpa_status gpa_rules_arrays(const gpa_rules* rules, uint64_t* n_rules, const uint32_t** itemset,
                                       const uint32_t** antecedent_mask, const uint32_t** antecedent_support) {
  return gpa::guard([&] {
    GPA_REQUIRE(rules, GPA_ERR_INVALID, "rules is NULL");
    const uint32_t* d = rules->data.p;
    if (n_rules) *n_rules = rules->n;
    if (itemset) *itemset = d;
    if (antecedent_mask) *antecedent_mask = d ? d + rules->n : nullptr;
    if (antecedent_support) *antecedent_support = d ? d + 2 * rules->n : nullptr;
  });
}

extern "C" gpa_status gpa_rules_destroy(gpa_rules* rules) {
  return gpa::guard([&] { delete rules; });
}
