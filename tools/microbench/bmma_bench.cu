// Microbenchmark: throughput and semantics of the binary tensor-core MMA
//   mma.sync.aligned.m16n8k256.row.col.s32.b1.b1.s32.and.popc
// on sm_100a: D[16x8] += popc(A[16x256 bits] AND B[256 bits x 8]) -- the paper's AND + popcount
// (P18@394) evaluated 32,768 cand.tx at a time.  Compares against the POPC pipe rate
// (profiles/r01_microbench_popc.txt).
#include <cstdio>
#include <cstdint>
#include <cstdlib>
#include <cuda_runtime.h>

__device__ __forceinline__ void bmma(uint32_t (&d)[4], const uint32_t (&a)[4], const uint32_t (&b)[2]) {
  asm volatile(
      "mma.sync.aligned.m16n8k256.row.col.s32.b1.b1.s32.and.popc {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, "
      "{%0,%1,%2,%3};"
      : "+r"(d[0]), "+r"(d[1]), "+r"(d[2]), "+r"(d[3])
      : "r"(a[0]), "r"(a[1]), "r"(a[2]), "r"(a[3]), "r"(b[0]), "r"(b[1]));
}

__device__ __forceinline__ void imma(uint32_t (&d)[4], const uint32_t (&a)[4], const uint32_t (&b)[2]) {
  asm volatile(
      "mma.sync.aligned.m16n8k32.row.col.s32.u8.u8.s32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, "
      "{%0,%1,%2,%3};"
      : "+r"(d[0]), "+r"(d[1]), "+r"(d[2]), "+r"(d[3])
      : "r"(a[0]), "r"(a[1]), "r"(a[2]), "r"(a[3]), "r"(b[0]), "r"(b[1]));
}
template <int NACC>
__global__ void imma_tput(const uint32_t* __restrict__ in, uint32_t* out, int iters) {
  uint32_t a[4], b[NACC][2], d[NACC][4];
  const int lane = threadIdx.x & 31;
#pragma unroll
  for (int i = 0; i < 4; ++i) a[i] = in[(lane * 4 + i) & 1023];
#pragma unroll
  for (int j = 0; j < NACC; ++j) {
    b[j][0] = in[(lane + 7 * j) & 1023];
    b[j][1] = in[(lane + 13 * j + 1) & 1023];
#pragma unroll
    for (int i = 0; i < 4; ++i) d[j][i] = 0;
  }
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int j = 0; j < NACC; ++j) imma(d[j], a, b[j]);
  }
  uint32_t s = 0;
#pragma unroll
  for (int j = 0; j < NACC; ++j) s += d[j][0] + d[j][1] + d[j][2] + d[j][3];
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}

// throughput: NACC independent accumulator tiles per warp
template <int NACC>
__global__ void bmma_tput(const uint32_t* __restrict__ in, uint32_t* out, int iters) {
  uint32_t a[4], b[NACC][2], d[NACC][4];
  const int lane = threadIdx.x & 31;
#pragma unroll
  for (int i = 0; i < 4; ++i) a[i] = in[(lane * 4 + i) & 1023];
#pragma unroll
  for (int j = 0; j < NACC; ++j) {
    b[j][0] = in[(lane + 7 * j) & 1023];
    b[j][1] = in[(lane + 13 * j + 1) & 1023];
#pragma unroll
    for (int i = 0; i < 4; ++i) d[j][i] = 0;
  }
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int j = 0; j < NACC; ++j) bmma(d[j], a, b[j]);
  }
  uint32_t s = 0;
#pragma unroll
  for (int j = 0; j < NACC; ++j) s += d[j][0] + d[j][1] + d[j][2] + d[j][3];
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}

// semantics: one warp, A = 16 rows x 256 bits (8 words per row), B = 8 rows x 256 bits,
// fragment layout assumed: a[0] = A[g][t], a[1] = A[g+8][t], a[2] = A[g][4+t], a[3] = A[g+8][4+t]
// (g = lane/4, t = lane%4, words of 32 bits); b[0] = B[g][t], b[1] = B[g][4+t];
// d[0..1] = D[g][2t..2t+1], d[2..3] = D[g+8][2t..2t+1].
__global__ void bmma_check(const uint32_t* A, const uint32_t* B, uint32_t* D) {
  const int lane = threadIdx.x, g = lane >> 2, t = lane & 3;
  uint32_t a[4] = {A[g * 8 + t], A[(g + 8) * 8 + t], A[g * 8 + 4 + t], A[(g + 8) * 8 + 4 + t]};
  uint32_t b[2] = {B[g * 8 + t], B[g * 8 + 4 + t]};
  uint32_t d[4] = {0, 0, 0, 0};
  bmma(d, a, b);
  D[g * 8 + 2 * t] = d[0];
  D[g * 8 + 2 * t + 1] = d[1];
  D[(g + 8) * 8 + 2 * t] = d[2];
  D[(g + 8) * 8 + 2 * t + 1] = d[3];
}

int main() {
  cudaDeviceProp prop;
  cudaGetDeviceProperties(&prop, 0);
  int clk;
  cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
  printf("%s SMs=%d clock_khz=%d\n", prop.name, prop.multiProcessorCount, clk);
  // --- semantics
  uint32_t hA[128], hB[64], hD[128];
  srand(1);
  for (auto& x : hA) x = (uint32_t)rand() * 2654435761u ^ rand();
  for (auto& x : hB) x = (uint32_t)rand() * 2246822519u ^ rand();
  uint32_t *dA, *dB, *dD;
  cudaMalloc(&dA, sizeof hA); cudaMalloc(&dB, sizeof hB); cudaMalloc(&dD, sizeof hD);
  cudaMemcpy(dA, hA, sizeof hA, cudaMemcpyHostToDevice);
  cudaMemcpy(dB, hB, sizeof hB, cudaMemcpyHostToDevice);
  bmma_check<<<1, 32>>>(dA, dB, dD);
  cudaError_t e = cudaDeviceSynchronize();
  if (e != cudaSuccess) { printf("check kernel failed: %s\n", cudaGetErrorString(e)); return 1; }
  cudaMemcpy(hD, dD, sizeof hD, cudaMemcpyDeviceToHost);
  int bad = 0;
  for (int m = 0; m < 16; ++m)
    for (int n = 0; n < 8; ++n) {
      uint32_t ref = 0;
      for (int w = 0; w < 8; ++w) ref += __builtin_popcount(hA[m * 8 + w] & hB[n * 8 + w]);
      if (ref != hD[m * 8 + n]) ++bad;
    }
  printf("semantics (assumed fragment layout): %d / 128 mismatches\n", bad);
  // --- throughput
  uint32_t *in, *out;
  cudaMalloc(&in, 4096); cudaMemset(in, 0x5a, 4096);
  const int threads = 256, iters = 4096;
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0); cudaEventCreate(&e1);
  for (int bps : {1, 2, 4, 8}) {
    const int blocks = prop.multiProcessorCount * bps;
    cudaMalloc(&out, (size_t)blocks * threads * 4);
    for (int rep = 0; rep < 2; ++rep) {
      cudaEventRecord(e0);
      bmma_tput<8><<<blocks, threads>>>(in, out, iters);
      cudaEventRecord(e1);
      cudaEventSynchronize(e1);
      float ms;
      cudaEventElapsedTime(&ms, e0, e1);
      const double mmas = (double)blocks * (threads / 32) * iters * 8;
      const double bitmacs = mmas * 16 * 8 * 256;
      if (rep)
        printf("blocks/SM=%d  %.3f ms  %.1f T bit-MAC/s (= cand.tx/s)  per-SM-per-clk(@%d MHz) = %.0f bit-MAC, %.2f clk per mma per SM\n",
               bps, ms, bitmacs / ms / 1e9, clk / 1000, bitmacs / (ms * 1e-3) / prop.multiProcessorCount / (clk * 1e3),
               (ms * 1e-3) * (clk * 1e3) * prop.multiProcessorCount / mmas);
    }
    cudaFree(out);
  }
  for (int bps : {2, 4}) {
    const int blocks = prop.multiProcessorCount * bps;
    cudaMalloc(&out, (size_t)blocks * threads * 4);
    for (int rep = 0; rep < 2; ++rep) {
      cudaEventRecord(e0);
      imma_tput<8><<<blocks, threads>>>(in, out, iters);
      cudaEventRecord(e1);
      cudaEventSynchronize(e1);
      float ms;
      cudaEventElapsedTime(&ms, e0, e1);
      const double mmas = (double)blocks * (threads / 32) * iters * 8;
      const double macs = mmas * 16 * 8 * 32;
      if (rep)
        printf("IMMA u8 m16n8k32 mma.sync: blocks/SM=%d %.3f ms  %.1f T int8-MAC/s  %.0f MAC/clk/SM\n", bps, ms,
               macs / ms / 1e9, macs / (ms * 1e-3) / prop.multiProcessorCount / (clk * 1e3));
    }
    cudaFree(out);
  }
  e = cudaDeviceSynchronize();
  printf("done: %s\n", cudaGetErrorString(e));
  return 0;
}
