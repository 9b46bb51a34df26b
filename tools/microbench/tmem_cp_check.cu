// Semantics check of tcgen05.cp.cta_group::1.32x128b.warpx4 (shared memory -> tensor memory,
// multicast to the 4 lane quarters) with a K-major no-swizzle source descriptor (8-row x 16-byte
// core matrices, SBO = 128 B), as count_trie_tm.cu uses it: source = 32 "rows" of 16 bytes at
// 16-byte stride (one 512-byte half of a 1 KB stripe segment), destination = 4 columns of every lane.
// Also times a 32-row stripe copy (64 copies) + commit round trip.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ uint64_t desc(uint32_t saddr) {
  return (uint64_t)((saddr >> 4) & 0x3fffu) | ((uint64_t)(16 >> 4) << 16) | ((uint64_t)(128 >> 4) << 32) | (1ull << 46);
}

__global__ void k(uint32_t* out, long long* cyc, int reps) {
  __shared__ __align__(1024) uint32_t seg[32 * 256];   // 32 rows x 1 KB
  __shared__ uint32_t s_t;
  __shared__ __align__(8) uint64_t bar;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  for (int i = threadIdx.x; i < 32 * 256; i += blockDim.x) seg[i] = 0x1000000u * (i / 256) + i % 256;  // row r, word w
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&bar)));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 256;" ::"r"(smem_u32(&s_t)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  const uint32_t t = s_t;
  long long c0 = 0, c1 = 0;
  if (threadIdx.x == 0) {
    c0 = clock64();
    for (int rep = 0; rep < reps; ++rep)
    for (int r = 0; r < 32; ++r)
      for (int h = 0; h < 2; ++h) {
        const uint64_t d = desc(smem_u32(seg) + r * 1024 + h * 512);
        asm volatile("tcgen05.cp.cta_group::1.32x128b.warpx4 [%0], %1;" ::"r"(t + 8 * r + 4 * h), "l"(d) : "memory");
      }
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(smem_u32(&bar))
                 : "memory");
  }
  __syncwarp();
  asm volatile(
      "{\n.reg .pred P1;\nW: mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], 0;\n@P1 bra D;\nbra W;\nD:\n}\n" ::"r"(
          smem_u32(&bar))
      : "memory");
  if (threadIdx.x == 0) c1 = clock64();
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  // every warp (lane quarter warp % 4) reads rows 0..31: 8 columns each
  int bad = 0;
  for (int r = 0; r < 32; ++r) {
    uint32_t v[8];
    asm volatile("tcgen05.ld.sync.aligned.32x32b.x8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                 : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7])
                 : "r"(t + ((uint32_t)((warp & 3) * 32) << 16) + 8 * r));
    asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
    for (int j = 0; j < 8; ++j) {
      const uint32_t w = (j < 4) ? 4 * lane + j : 128 + 4 * lane + (j - 4);
      if (v[j] != 0x1000000u * r + w) ++bad;
    }
  }
  out[threadIdx.x] = bad;
  if (threadIdx.x == 0) *cyc = c1 - c0;
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 256;" ::"r"(t));
}

// .128x256b: lane i <- 32 bytes (chunk 0 at +16 i, chunk 1 at +2048 + 16 i) of a 4 KB "row segment"
__device__ __forceinline__ uint64_t desc2(uint32_t saddr) {
  return (uint64_t)((saddr >> 4) & 0x3fffu) | ((uint64_t)(2048 >> 4) << 16) | ((uint64_t)(128 >> 4) << 32) |
         (1ull << 46);
}
__global__ void k2(uint32_t* out, long long* cyc, int reps) {
  __shared__ __align__(1024) uint32_t seg[8 * 1024];   // 8 rows x 4 KB
  __shared__ uint32_t s_t;
  __shared__ __align__(8) uint64_t bar;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  for (int i = threadIdx.x; i < 8 * 1024; i += blockDim.x) seg[i] = 0x1000000u * (i / 1024) + i % 1024;
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&bar)));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 256;" ::"r"(smem_u32(&s_t)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  const uint32_t t = s_t;
  long long c0 = 0, c1 = 0;
  if (threadIdx.x == 0) {
    c0 = clock64();
    for (int rep = 0; rep < reps; ++rep)
      for (int r = 0; r < 32; ++r)
        asm volatile("tcgen05.cp.cta_group::1.128x256b [%0], %1;" ::"r"(t + 8 * r), "l"(desc2(smem_u32(seg) + (r & 7) * 4096))
                     : "memory");
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(smem_u32(&bar))
                 : "memory");
  }
  __syncwarp();
  asm volatile(
      "{\n.reg .pred P1;\nW: mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], 0;\n@P1 bra D;\nbra W;\nD:\n}\n" ::"r"(
          smem_u32(&bar))
      : "memory");
  if (threadIdx.x == 0) c1 = clock64();
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  int bad = 0;
  const int q = warp & 3;
  for (int r = 0; r < 32; ++r) {
    uint32_t v[8];
    asm volatile("tcgen05.ld.sync.aligned.32x32b.x8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                 : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7])
                 : "r"(t + ((uint32_t)(q * 32) << 16) + 8 * r));
    asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
    for (int j = 0; j < 8; ++j) {
      // lane i = 32 q + lane: chunk 0 at byte 16 i -> words 4 i..4 i+3, chunk 1 at 2048 + 16 i
      const uint32_t i = 32 * q + lane;
      const uint32_t w = (j < 4) ? 4 * i + j : 512 + 4 * i + (j - 4);
      if (v[j] != 0x1000000u * (r & 7) + w) ++bad;
    }
  }
  out[threadIdx.x] = bad;
  if (threadIdx.x == 0) *cyc = c1 - c0;
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 256;" ::"r"(t));
}

int main() {
  uint32_t* out;
  long long* cyc;
  cudaMalloc(&out, 256 * 4);
  cudaMalloc(&cyc, 8);
  for (int reps : {1, 1, 2, 4, 16}) {
  k<<<1, 256>>>(out, cyc, reps);
  cudaError_t e = cudaDeviceSynchronize();
  if (e != cudaSuccess) { printf("error %s\n", cudaGetErrorString(e)); return 1; }
  uint32_t h[256];
  long long c;
  cudaMemcpy(h, out, sizeof h, cudaMemcpyDeviceToHost);
  cudaMemcpy(&c, cyc, 8, cudaMemcpyDeviceToHost);
  long long tot = 0;
  for (int i = 0; i < 256; ++i) tot += h[i];
  printf("tcgen05.cp 32x128b.warpx4: %lld mismatching words over 8 warps x 32 rows x 8 words; %d x 64 copies + commit = %lld clk\n",
         tot, reps, c);
  }
  for (int reps : {1, 4, 16}) {
    k2<<<1, 256>>>(out, cyc, reps);
    cudaError_t e = cudaDeviceSynchronize();
    if (e != cudaSuccess) { printf("error %s\n", cudaGetErrorString(e)); return 1; }
    uint32_t h[256];
    long long c;
    cudaMemcpy(h, out, sizeof h, cudaMemcpyDeviceToHost);
    cudaMemcpy(&c, cyc, 8, cudaMemcpyDeviceToHost);
    long long tot = 0;
    for (int i = 0; i < 256; ++i) tot += h[i];
    printf("tcgen05.cp 128x256b (LBO 2 KB): %lld mismatching words; %d x 32 copies (4 KB each) + commit = %lld clk\n",
           tot, reps, c);
  }
  return 0;
}
