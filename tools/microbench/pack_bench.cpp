#include <chrono>
#include <cstdio>
#include <cstdint>
#include <vector>
#include <thread>
#include <random>
#include <array>
#include <utility>
template <uint32_t B>
inline uint32_t pack_block(const uint32_t* __restrict__ src, uint32_t* __restrict__ dst) {
  uint32_t orv = 0; uint64_t acc = 0; uint32_t nb = 0, k = 0;
#pragma GCC unroll 32
  for (uint32_t i = 0; i < 32; ++i) { const uint32_t v = src[i]; orv |= v; acc |= (uint64_t)v << nb; nb += B;
    if (nb >= 32) { dst[k++] = (uint32_t)acc; acc >>= 32; nb -= 32; } }
  return orv;
}
int main() {
  const uint64_t n = 420000000ull / 8;  // per-thread share of 8 threads
  int T = std::thread::hardware_concurrency();
  std::vector<uint32_t> items(n * T); std::vector<uint32_t> out(n * T / 32 * 10 + 16);
  for (size_t i = 0; i < items.size(); ++i) items[i] = (i * 2654435761u) % 1000;
  for (int rep = 0; rep < 3; ++rep) {
    auto t0 = std::chrono::steady_clock::now();
    std::vector<std::thread> th;
    for (int t = 0; t < T; ++t) th.emplace_back([&, t] { uint32_t o = 0; for (uint64_t b = t * (n / 32); b < (t + 1) * (n / 32); ++b) o |= pack_block<10>(&items[b * 32], &out[b * 10]); if (o == 12345) printf("x"); });
    for (auto& x : th) x.join();
    double ms = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
    printf("threads %d: %.1f ms for %.2f GB of u32 (%.1f GB/s)\n", T, ms, n * T * 4 / 1e9, n * T * 4 / 1e6 / ms);
  }
}
