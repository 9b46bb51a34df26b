// Microbenchmark: POPC / LOP3 / IADD throughput per SM on sm_100a, and streaming read bandwidth.
// Used to derive the ALU roofline for the support-counting kernels.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

template <int MODE>
__global__ void alu_kernel(const uint32_t* __restrict__ in, uint32_t* out, int iters) {
  uint32_t a[16], acc[16];
#pragma unroll
  for (int i = 0; i < 16; ++i) { a[i] = in[(threadIdx.x + i) & 255] ^ (i * 0x9e3779b9u); acc[i] = 0; }
  uint32_t m = in[threadIdx.x & 255];
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int i = 0; i < 16; ++i) {
      if (MODE == 0) {            // popc only (+ add)
        acc[i] += __popc(a[i] ^ acc[i]);
      } else if (MODE == 1) {     // and + popc + add : the counting inner op
        acc[i] += __popc(a[i] & m);
        a[i] = a[i] * 0 + (a[i] ^ it);
      } else {                    // pure LOP3 chain
        acc[i] = (acc[i] & a[i]) ^ (m | acc[i]) ^ it;
      }
    }
  }
  uint32_t s = 0;
#pragma unroll
  for (int i = 0; i < 16; ++i) s += acc[i];
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}

__global__ void read_kernel(const uint4* __restrict__ p, size_t n, uint32_t* out) {
  uint32_t s = 0;
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x) {
    uint4 v = __ldg(p + i);
    s += __popc(v.x) + __popc(v.y) + __popc(v.z) + __popc(v.w);
  }
  if (s == 0xdeadbeef) out[0] = s;
}

int main() {
  int dev = 0; cudaDeviceProp prop; cudaGetDeviceProperties(&prop, dev);
  int clk; cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, dev);
  printf("%s SMs=%d clock_khz=%d l2=%d\n", prop.name, prop.multiProcessorCount, clk, prop.l2CacheSize);
  uint32_t *in, *out; cudaMalloc(&in, 1024 * 4); cudaMemset(in, 0x5a, 4096);
  int blocks = prop.multiProcessorCount * 8, threads = 256, iters = 4096;
  cudaMalloc(&out, (size_t)blocks * threads * 4);
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  const char* names[3] = {"popc+add", "and+popc+add", "lop3x3"};
  for (int mode = 0; mode < 3; ++mode) {
    for (int rep = 0; rep < 3; ++rep) {
      cudaEventRecord(e0);
      if (mode == 0) alu_kernel<0><<<blocks, threads>>>(in, out, iters);
      if (mode == 1) alu_kernel<1><<<blocks, threads>>>(in, out, iters);
      if (mode == 2) alu_kernel<2><<<blocks, threads>>>(in, out, iters);
      cudaEventRecord(e1); cudaEventSynchronize(e1);
      float ms; cudaEventElapsedTime(&ms, e0, e1);
      double ops = (double)blocks * threads * iters * 16;
      if (rep == 2) printf("%-14s %.3f ms  %.3f Gop/s  per-SM-per-clk(@max %d MHz)=%.2f\n", names[mode], ms, ops / ms / 1e6,
             clk / 1000, ops / (ms * 1e-3) / prop.multiProcessorCount / (clk * 1e3));
    }
  }
  size_t bytes = (size_t)4 << 30; uint4* big; cudaMalloc(&big, bytes); cudaMemset(big, 1, bytes);
  for (int rep = 0; rep < 4; ++rep) {
    cudaEventRecord(e0);
    read_kernel<<<prop.multiProcessorCount * 16, 512>>>(big, bytes / 16, out);
    cudaEventRecord(e1); cudaEventSynchronize(e1);
    float ms; cudaEventElapsedTime(&ms, e0, e1);
    printf("read+popc 4GiB: %.3f ms  %.1f GB/s\n", ms, bytes / ms / 1e6);
  }
  printf("err=%s\n", cudaGetErrorString(cudaGetLastError()));
  return 0;
}
