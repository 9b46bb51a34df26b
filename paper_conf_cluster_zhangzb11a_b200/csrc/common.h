// Internal helpers shared by the library's runtime (.cpp) and kernel (.cu) translation units.
// Nothing here is part of the C ABI (include/gpapriori.h is).
#pragma once
#include <atomic>
#include <mutex>
#include <map>
#include <cstdint>
#include <cstdio>
#include <string>
#include <utility>
#include <cuda_runtime.h>
#include "gpapriori.h"

namespace gpa {

// Process-wide count of the library's kernel launches (every <<<>>> site and CUB's scan kernels),
// exported through gpa_kernel_launches() so a benchmark can state how many of its kernels ran.
inline std::atomic<uint64_t> g_kernel_launches{0};
inline void note_launch(uint64_t n = 1) { g_kernel_launches.fetch_add(n, std::memory_order_relaxed); }

struct Error {
  gpa_status status;
  std::string msg;
};

[[noreturn]] void fail(gpa_status st, const char* fmt, ...) __attribute__((format(printf, 2, 3)));
// cudaStreamSynchronize, except inside a collective call (DistScope, runtime/context.cpp): then it
// polls the communicator for asynchronous errors and times out instead of hanging on a lost peer.
void stream_wait(cudaStream_t s);
bool trace_enabled();   // GPA_TRACE=1 (runtime/context.cpp)
double wall_ms();       // host steady clock, ms
void set_last_error(gpa_status st, const std::string& msg);

#define GPA_CUDA(call)                                                                              \
  do {                                                                                              \
    cudaError_t e_ = (call);                                                                        \
    if (e_ != cudaSuccess)                                                                          \
      ::gpa::fail(GPA_ERR_CUDA, "%s failed: %s (%s:%d)", #call, cudaGetErrorString(e_), __FILE__, __LINE__); \
  } while (0)

#define GPA_REQUIRE(cond, st, ...)                                                                  \
  do {                                                                                              \
    if (!(cond)) ::gpa::fail(st, __VA_ARGS__);                                                      \
  } while (0)

// Row layout of the static bitset: pitch (in 32-bit words) is a multiple of this many words
// (4 KB = 32,768 transactions).  The paper aligns rows to 64 bytes (P18@1685); 4 KB is a whole
// number of 128-B L2 lines / TMA boxes (pair kernels) and of every trie stripe (128 / 256 words
// in shared memory, 1,024 words in tensor memory), so no kernel ever handles a ragged row tail.
constexpr uint64_t kPitchWords = 1024;

inline uint64_t pitch_words_for(uint64_t n_tx) {
  uint64_t w = (n_tx + 31) / 32;
  w = (w + kPitchWords - 1) / kPitchWords * kPitchWords;
  return w ? w : kPitchWords;
}

// Index of pair (a, b), a < b, among all pairs of n rows in lexicographic order.
__host__ __device__ inline uint64_t pair_index(uint64_t a, uint64_t b, uint64_t n) {
  return a * n - a * (a + 1) / 2 + (b - a - 1);
}

// Device buffer allocated from the device's stream-ordered pool (cudaMallocAsync).  The pool's
// release threshold is raised once per device so repeated calls reuse memory without a
// cudaMalloc / cudaFree round trip.
template <class T>
struct DBuf {
  T* p = nullptr;
  size_t n = 0;
  cudaStream_t s = nullptr;
  DBuf() = default;
  DBuf(const DBuf&) = delete;
  DBuf& operator=(const DBuf&) = delete;
  DBuf(DBuf&& o) noexcept { swap(o); }
  DBuf& operator=(DBuf&& o) noexcept { reset(); swap(o); return *this; }
  ~DBuf() { reset(); }
  void swap(DBuf& o) noexcept { std::swap(p, o.p); std::swap(n, o.n); std::swap(s, o.s); }
  void reset() noexcept {
    if (p) cudaFreeAsync(p, s);
    p = nullptr; n = 0;
  }
  void alloc(size_t count, cudaStream_t stream) {
    reset();
    s = stream;
    n = count;
    if (count == 0) return;
    cudaError_t e = cudaMallocAsync(reinterpret_cast<void**>(&p), count * sizeof(T), stream);
    if (e != cudaSuccess) {
      p = nullptr;
      n = 0;
      cudaGetLastError();
      fail(e == cudaErrorMemoryAllocation ? GPA_ERR_OOM : GPA_ERR_CUDA, "device allocation of %zu bytes failed: %s",
           count * sizeof(T), cudaGetErrorString(e));
    }
  }
  // grow-only reuse
  void ensure(size_t count, cudaStream_t stream) {
    if (count > n || stream != s) alloc(count, stream);
  }
};

// Persistent grow-only device buffer (cudaMalloc / cudaFree, not stream-ordered): for the large
// per-generation workspaces (projected lists) that a stream-ordered pool would re-map on every
// call -- measured: cudaMallocAsync of 0.7 GB blocking the host for up to 0.5 s once the pool
// fragments.  Grows by 1.25x so that a sequence of mining calls settles on one allocation.
template <class T>
struct PBuf {
  T* p = nullptr;
  size_t n = 0;
  PBuf() = default;
  PBuf(const PBuf&) = delete;
  PBuf& operator=(const PBuf&) = delete;
  ~PBuf() {
    if (p) cudaFree(p);
  }
  T* ensure(size_t count) {
    if (count == 0) count = 1;
    if (count <= n) return p;
    if (p) cudaFree(p);  // synchronises: no kernel still reads the old buffer
    p = nullptr;
    n = 0;
    const size_t want = count + count / 4;
    cudaError_t e = cudaMalloc(reinterpret_cast<void**>(&p), want * sizeof(T));
    if (e != cudaSuccess) {
      p = nullptr;
      cudaGetLastError();
      fail(e == cudaErrorMemoryAllocation ? GPA_ERR_OOM : GPA_ERR_CUDA, "device allocation of %zu bytes failed: %s",
           want * sizeof(T), cudaGetErrorString(e));
    }
    n = want;
    return p;
  }
};

// cudaFuncAttributeMaxDynamicSharedMemorySize is a per-DEVICE attribute of a kernel: raise it
// per (kernel, device) to the largest size requested so far, under a lock (a second device or a
// concurrent thread must not launch without it; a smaller request never lowers it).
inline void ensure_smem_attr(const void* func, int bytes) {
  static std::mutex mu;
  static std::map<std::pair<const void*, int>, int> set_to;
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess) fail(GPA_ERR_CUDA, "cudaGetDevice failed");
  std::lock_guard<std::mutex> lk(mu);
  int& cur = set_to[std::make_pair(func, dev)];
  if (bytes <= cur) return;
  cudaError_t e = cudaFuncSetAttribute(func, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes);
  if (e != cudaSuccess) fail(GPA_ERR_CUDA, "cudaFuncSetAttribute failed: %s", cudaGetErrorString(e));
  cur = bytes;
}

// Flags written by the validation/histogram kernel.
constexpr uint32_t kFlagBadOffsets = 1u;
constexpr uint32_t kFlagBadItem = 2u;
constexpr uint32_t kFlagNonCanonical = 4u;

}  // namespace gpa
