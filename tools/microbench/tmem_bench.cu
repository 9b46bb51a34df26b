// Microbenchmark: tensor-memory read bandwidth (tcgen05.ld.32x32b.xN into registers) vs
// shared-memory LDS.128, per SM on sm_100a -- can TMEM serve the trie kernel's row words
// (count_trie.cu is bound by shared-memory wavefronts) faster than shared memory?
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

template <int X>
__device__ __forceinline__ void tld(uint32_t (&v)[8], uint32_t addr);
template <>
__device__ __forceinline__ void tld<8>(uint32_t (&v)[8], uint32_t addr) {
  asm volatile("tcgen05.ld.sync.aligned.32x32b.x8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
               : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7])
               : "r"(addr));
}

// WAVE loads in flight before each wait
template <int WAVE>
__global__ void __launch_bounds__(512, 1) tmem_kernel(uint32_t* out, int iters, int mode) {
  __shared__ uint32_t s_t;
  __shared__ __align__(16) uint32_t sm[8 * 1024];   // 32 KB for the LDS comparison
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(
        (uint32_t)__cvta_generic_to_shared(&s_t)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  for (int i = threadIdx.x; i < 8 * 1024; i += blockDim.x) sm[i] = i * 2654435761u;
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  const uint32_t t = s_t;
  const uint32_t q = (warp & 3) * 32;
  // fill: each warp of quarter 0..3 writes its lanes (warps 0-3 only)
  if (warp < 4) {
    for (int c = 0; c < 512; c += 8) {
      uint32_t w[8];
      for (int j = 0; j < 8; ++j) w[j] = (lane + 1) * 7919u + c + j;
      asm volatile("tcgen05.st.sync.aligned.32x32b.x8.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};" ::"r"(t + (q << 16) + c),
                   "r"(w[0]), "r"(w[1]), "r"(w[2]), "r"(w[3]), "r"(w[4]), "r"(w[5]), "r"(w[6]), "r"(w[7]));
    }
    asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  uint32_t acc8[8] = {0, 0, 0, 0, 0, 0, 0, 0}, col = (warp * 40) & 511;
  if (mode == 0) {
    for (int it = 0; it < iters; ++it) {
      uint32_t v[WAVE][8];
#pragma unroll
      for (int u = 0; u < WAVE; ++u) tld<8>(v[u], t + (q << 16) + ((col + u * 72) & 504));
      asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
#pragma unroll
      for (int u = 0; u < WAVE; ++u)
#pragma unroll
        for (int j = 0; j < 8; j += 8)
          acc8[u & 7] ^= (v[u][0] ^ v[u][1] ^ v[u][2]) ^ (v[u][3] ^ v[u][4] ^ v[u][5]) ^ (v[u][6] ^ v[u][7]);
      col += 136;
    }
  } else if (mode == 2) {
    const uint32_t base = (uint32_t)__cvta_generic_to_shared(sm) + lane * 16;
    for (int it = 0; it < iters; ++it) {
      uint32_t v[WAVE / 2][8];
#pragma unroll
      for (int u = 0; u < WAVE / 2; ++u) tld<8>(v[u], t + (q << 16) + ((col + u * 72) & 504));
#pragma unroll
      for (int u = WAVE / 2; u < WAVE; ++u) {
        uint4 a, b;
        const uint32_t ad = base + (((col + u * 72) & 31) * 1024);
        asm volatile("ld.shared.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(a.x), "=r"(a.y), "=r"(a.z), "=r"(a.w) : "r"(ad));
        asm volatile("ld.shared.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(b.x), "=r"(b.y), "=r"(b.z), "=r"(b.w) : "r"(ad + 512));
        acc8[u & 7] ^= (a.x ^ a.y ^ a.z) ^ (a.w ^ b.x ^ b.y) ^ (b.z ^ b.w);
      }
      asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
#pragma unroll
      for (int u = 0; u < WAVE / 2; ++u)
        acc8[u & 7] ^= (v[u][0] ^ v[u][1] ^ v[u][2]) ^ (v[u][3] ^ v[u][4] ^ v[u][5]) ^ (v[u][6] ^ v[u][7]);
      col += 136;
    }
  } else {
    const uint32_t base = (uint32_t)__cvta_generic_to_shared(sm) + lane * 16;
    for (int it = 0; it < iters; ++it) {
#pragma unroll
      for (int u = 0; u < WAVE; ++u) {
        uint4 a, b;
        const uint32_t ad = base + (((col + u * 72) & 31) * 1024);
        asm volatile("ld.shared.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(a.x), "=r"(a.y), "=r"(a.z), "=r"(a.w) : "r"(ad));
        asm volatile("ld.shared.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(b.x), "=r"(b.y), "=r"(b.z), "=r"(b.w) : "r"(ad + 512));
        acc8[u & 7] ^= (a.x ^ a.y ^ a.z) ^ (a.w ^ b.x ^ b.y) ^ (b.z ^ b.w);
      }
      col += 136;
    }
  }
  uint32_t acc = 0;
#pragma unroll
  for (int j = 0; j < 8; ++j) acc += acc8[j];
  out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(t));
}

int main() {
  cudaDeviceProp prop;
  cudaGetDeviceProperties(&prop, 0);
  int clk;
  cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
  printf("%s SMs=%d clock_khz=%d\n", prop.name, prop.multiProcessorCount, clk);
  uint32_t* out;
  const int blocks = prop.multiProcessorCount, iters = 20000;
  cudaMalloc(&out, (size_t)blocks * 512 * 4);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  for (int wave : {4, 8})
  for (int threads : {128, 256, 512})
    for (int mode = 0; mode < 3; ++mode)
      for (int rep = 0; rep < 2; ++rep) {
        cudaEventRecord(e0);
        if (wave == 4) tmem_kernel<4><<<blocks, threads>>>(out, iters, mode);
        else tmem_kernel<8><<<blocks, threads>>>(out, iters / 2, mode);
        cudaEventRecord(e1);
        cudaError_t e = cudaEventSynchronize(e1);
        if (e != cudaSuccess) { printf("error %s\n", cudaGetErrorString(e)); return 1; }
        float ms;
        cudaEventElapsedTime(&ms, e0, e1);
        // bytes moved into registers: per warp-iteration 4 loads x 32 lanes x 32 B
        const double bytes = (double)blocks * (threads / 32) * iters * 4 * 32 * 32;
        if (rep)
          printf("wave=%d %s threads=%3d  %.3f ms  %.0f B/clk/SM  (%.1f TB/s total)\n",
                 wave, mode == 1 ? "LDS.128 x2   " : mode == 2 ? "half+half    " : "tcgen05.ld x8", threads, ms,
                 bytes / (ms * 1e-3) / blocks / (clk * 1e3), bytes / ms / 1e9);
      }
  return 0;
}
