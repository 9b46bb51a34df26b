// Association rules from a mining result (gpa_rules_*, Q19): the
// result's frequent itemsets go to the device once, the rules are enumerated there (rules.cu)
// and come back as three arrays owned by the gpa_rules handle.
#include <algorithm>

#include "internal.h"

struct gpa_rules {
  std::vector<uint32_t> itemset, mask, supp_a;
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
      device_rules(d_items.p, d_off.p, d_len.p, d_sup.p, (uint32_t)n, (uint32_t)x0, conf_num, conf_den, di.n_sms, s,
                   R->itemset, R->mask, R->supp_a);
    }
    *out = R;
    g.p = nullptr;
  });
}

extern "C" gpa_status gpa_rules_arrays(const gpa_rules* rules, uint64_t* n_rules, const uint32_t** itemset,
                                       const uint32_t** antecedent_mask, const uint32_t** antecedent_support) {
  return gpa::guard([&] {
    GPA_REQUIRE(rules, GPA_ERR_INVALID, "rules is NULL");
    if (n_rules) *n_rules = rules->itemset.size();
    if (itemset) *itemset = rules->itemset.data();
    if (antecedent_mask) *antecedent_mask = rules->mask.data();
    if (antecedent_support) *antecedent_support = rules->supp_a.data();
  });
}

extern "C" gpa_status gpa_rules_destroy(gpa_rules* rules) {
  return gpa::guard([&] { delete rules; });
}
