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
