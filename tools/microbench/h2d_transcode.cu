// Would narrowing the item ids on the host (u32 -> u16, item ids < 65,536) shorten the PCIe upload of
// the CSR?  (a) H2D of the u32 items from pinned memory, (b) the host conversion alone on T threads,
// (c) conversion of chunk c+1 pipelined with the H2D of chunk c (u16).
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -Xcompiler -fopenmp -o tools/microbench/h2d_transcode \
//        tools/microbench/h2d_transcode.cu
#include <cuda_runtime.h>
#include <omp.h>
#include <chrono>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <cstring>

#define CK(x)                                                                    \
  do {                                                                           \
    cudaError_t e = (x);                                                         \
    if (e != cudaSuccess) {                                                      \
      fprintf(stderr, "%s:%d %s\n", __FILE__, __LINE__, cudaGetErrorString(e));  \
      exit(1);                                                                   \
    }                                                                            \
  } while (0)

static double now_ms() {
  return std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now().time_since_epoch()).count();
}

static void narrow(const uint32_t* src, uint16_t* dst, size_t n) {
#pragma omp parallel for schedule(static)
  for (long long i = 0; i < (long long)n; ++i) dst[i] = (uint16_t)src[i];
}

int main() {
  const size_t n = 400ull << 20;   // 419 M items = 1.68 GB (T40I10D10M has 393 M)
  const int chunks = 8;
  const size_t cn = n / chunks;
  uint32_t* src;
  uint16_t* stage[2];
  CK(cudaHostAlloc(&src, n * 4, cudaHostAllocDefault));
  for (auto& p : stage) CK(cudaHostAlloc(&p, cn * 2, cudaHostAllocDefault));
#pragma omp parallel for
  for (long long i = 0; i < (long long)n; ++i) src[i] = (uint32_t)((i * 2654435761ull) % 1000);
  uint32_t* d32;
  uint16_t* d16;
  CK(cudaMalloc(&d32, n * 4));
  CK(cudaMalloc(&d16, n * 2));
  cudaStream_t s;
  CK(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
  cudaEvent_t done[2];
  for (auto& ev : done) CK(cudaEventCreateWithFlags(&ev, cudaEventDisableTiming));
  printf("threads %d\n", omp_get_max_threads());
  for (int rep = 0; rep < 3; ++rep) {
    double t0 = now_ms();
    CK(cudaMemcpyAsync(d32, src, n * 4, cudaMemcpyHostToDevice, s));
    CK(cudaStreamSynchronize(s));
    double t1 = now_ms();
    printf("(a) H2D u32 %.1f MB: %.2f ms = %.1f GB/s\n", n * 4 / 1e6, t1 - t0, n * 4 / 1e6 / (t1 - t0));
    t0 = now_ms();
    for (int c = 0; c < chunks; ++c) narrow(src + c * cn, stage[c & 1], cn);
    t1 = now_ms();
    printf("(b) narrow alone: %.2f ms = %.1f GB/s of u32 input\n", t1 - t0, n * 4 / 1e6 / (t1 - t0));
    t0 = now_ms();
    for (int c = 0; c < chunks; ++c) {
      if (c >= 2) CK(cudaEventSynchronize(done[c & 1]));   // staging buffer free again
      narrow(src + c * cn, stage[c & 1], cn);
      CK(cudaMemcpyAsync(d16 + c * cn, stage[c & 1], cn * 2, cudaMemcpyHostToDevice, s));
      CK(cudaEventRecord(done[c & 1], s));
    }
    CK(cudaStreamSynchronize(s));
    t1 = now_ms();
    printf("(c) narrow + H2D u16 pipelined: %.2f ms (%.1f GB/s of u32 input)\n", t1 - t0, n * 4 / 1e6 / (t1 - t0));
  }
  return 0;
}
