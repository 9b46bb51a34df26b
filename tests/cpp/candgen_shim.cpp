// Test shim (CPU only): exposes the GPU path's host candidate generation (runtime/candgen.cpp)
// through a plain C function so tests/test_host_logic.py can compare it with the oracle's
// independent implementation.  Not part of the library or its ABI.
#include <cstring>
#include <vector>
#include "runtime/internal.h"

extern "C" int shim_candgen(const uint32_t* L, uint64_t n, uint32_t km1, uint32_t* prefix_out, uint64_t* ext_off_out,
                            uint32_t* ext_out, uint64_t cap, uint64_t* n_groups, uint64_t* n_cand) {
  std::vector<uint32_t> v(L, L + n * km1);
  gpa::GroupedBatch b = gpa::candgen_join_prune(v, n, km1);
  *n_groups = b.groups();
  *n_cand = b.size();
  if (b.size() > cap || b.groups() > cap) return 1;
  if (!b.prefix.empty()) memcpy(prefix_out, b.prefix.data(), b.prefix.size() * 4);
  memcpy(ext_off_out, b.ext_off.data(), b.ext_off.size() * 8);
  if (!b.ext.empty()) memcpy(ext_out, b.ext.data(), b.ext.size() * 4);
  return 0;
}

// plan_trie of the join of L: writes blocks (4 u32 each), rows, lrows (16 B each), lcp.
extern "C" int shim_plan_trie(const uint32_t* L, uint64_t n, uint32_t km1, uint32_t n_rows, uint32_t* blocks_out,
                              uint64_t* n_blocks, uint32_t* rows_out, uint64_t* n_rows_out, uint8_t* lrows_out,
                              uint8_t* lcp_out, uint32_t* cand_out, uint64_t cap, uint64_t* n_cand) {
  std::vector<uint32_t> v(L, L + n * km1);
  gpa::GroupedBatch b = gpa::candgen_join_prune(v, n, km1);
  gpa::TriePlan P = gpa::plan_trie(b, n_rows);
  *n_blocks = P.blocks.size();
  *n_rows_out = P.rows.size();
  *n_cand = b.size();
  if (b.size() > cap || P.rows.size() > cap || P.blocks.size() > cap) return 1;
  memcpy(blocks_out, P.blocks.data(), P.blocks.size() * sizeof(gpa::TrieBlock));
  memcpy(rows_out, P.rows.data(), P.rows.size() * 4);
  memcpy(lrows_out, P.lrows.data(), P.lrows.size() * 16);
  memcpy(lcp_out, P.lcp.data(), P.lcp.size());
  const uint32_t k = km1 + 1;
  for (uint64_t g = 0; g < b.groups(); ++g)
    for (uint64_t j = b.ext_off[g]; j < b.ext_off[g + 1]; ++j) {
      for (uint32_t d = 0; d < km1; ++d) cand_out[j * k + d] = b.prefix[g * km1 + d];
      cand_out[j * k + km1] = b.ext[j];
    }
  return 0;
}
