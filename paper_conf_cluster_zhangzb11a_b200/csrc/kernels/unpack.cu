// Item ids of a host CSR chunk uploaded bit-packed (runtime/ingest.cpp): item j of the chunk sits
// at bit j * bits of a little-endian stream of 32-bit words (bits = ceil(log2 n_items) <= 16), so
// the PCIe transfer -- the end-to-end bound of gpa_mine on host input -- carries bits / 32 of the
// bytes.  One thread per item, widened back to u32 in place in the device CSR.  Exact (a bit copy).
#include <cstdint>

#include "../common.h"
#include "../kernels.h"

namespace gpa {
namespace {

__global__ void unpack_items_kernel(const uint32_t* __restrict__ packed, uint64_t n, uint32_t bits,
                                    uint32_t* __restrict__ out) {
  const uint32_t mask = (1u << bits) - 1u;
  for (uint64_t j = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; j < n; j += (uint64_t)gridDim.x * blockDim.x) {
    const uint64_t bit = j * bits;
    const uint64_t w = bit >> 5;
    const uint32_t s = (uint32_t)(bit & 31);
    uint32_t v = __ldg(packed + w) >> s;
    if (s + bits > 32) v |= __ldg(packed + w + 1) << (32 - s);
    out[j] = v & mask;
  }
}

}  // namespace

void launch_unpack_items(const uint32_t* packed, uint64_t n, uint32_t bits, uint32_t* out, int n_sms,
                         cudaStream_t stream) {
  if (n == 0) return;
  GPA_REQUIRE(bits >= 1 && bits <= 16, GPA_ERR_INVALID, "unpack: %u bits per item", bits);
  uint64_t g = (n + 255) / 256;
  const uint64_t cap = (uint64_t)n_sms * 16;
  if (g > cap) g = cap;
  { unpack_items_kernel<<<(unsigned)g, 256, 0, stream>>>(packed, n, bits, out); note_launch(); }
  GPA_CUDA(cudaGetLastError());
}

}  // namespace gpa
