// Launch-to-launch gap of small dependent kernels on one stream, with and without programmatic
// dependent launch (PDL), and the host round trip of "kernel -> sizes to the host -> host reacts"
// by (a) cudaMemcpyAsync D2H + cudaStreamSynchronize and (b) a kernel writing mapped pinned memory
// that the host polls.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/microbench/launch_gap tools/microbench/launch_gap.cu
#include <cuda_runtime.h>
#include <chrono>
#include <cstdio>
#include <cstdlib>

#define CK(x)                                                                    \
  do {                                                                           \
    cudaError_t e = (x);                                                         \
    if (e != cudaSuccess) {                                                      \
      fprintf(stderr, "%s:%d %s\n", __FILE__, __LINE__, cudaGetErrorString(e));  \
      exit(1);                                                                   \
    }                                                                            \
  } while (0)

__global__ void tiny(unsigned* p, unsigned n) {
  const unsigned i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i < n) p[i] += 1;
}

__global__ void tiny_pdl(unsigned* p, unsigned n) {
  asm volatile("griddepcontrol.wait;" ::: "memory");
  const unsigned i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i < n) p[i] += 1;
  asm volatile("griddepcontrol.launch_dependents;");
}

__global__ void sizes_to_host(const unsigned* p, volatile unsigned* host, unsigned seq) {
  if (threadIdx.x == 0) {
    host[1] = p[0];
    __threadfence_system();
    host[0] = seq;
  }
}

static double now_us() {
  return std::chrono::duration<double, std::micro>(std::chrono::steady_clock::now().time_since_epoch()).count();
}

int main() {
  const int iters = 2000;
  unsigned* d;
  CK(cudaMalloc(&d, 1 << 20));
  CK(cudaMemset(d, 0, 1 << 20));
  cudaStream_t s;
  CK(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
  cudaEvent_t a, b;
  CK(cudaEventCreate(&a));
  CK(cudaEventCreate(&b));
  for (unsigned blocks : {1u, 148u, 592u}) {
    const unsigned n = blocks * 256;
    for (int w = 0; w < 100; ++w) tiny<<<blocks, 256, 0, s>>>(d, n);
    CK(cudaEventRecord(a, s));
    for (int i = 0; i < iters; ++i) tiny<<<blocks, 256, 0, s>>>(d, n);
    CK(cudaEventRecord(b, s));
    CK(cudaEventSynchronize(b));
    float ms;
    CK(cudaEventElapsedTime(&ms, a, b));
    printf("plain launch, %4u blocks: %.2f us per dependent kernel\n", blocks, ms * 1e3 / iters);

    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(blocks);
    cfg.blockDim = dim3(256);
    cfg.stream = s;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    for (int w = 0; w < 100; ++w) CK(cudaLaunchKernelEx(&cfg, tiny_pdl, d, n));
    CK(cudaEventRecord(a, s));
    for (int i = 0; i < iters; ++i) CK(cudaLaunchKernelEx(&cfg, tiny_pdl, d, n));
    CK(cudaEventRecord(b, s));
    CK(cudaEventSynchronize(b));
    CK(cudaEventElapsedTime(&ms, a, b));
    printf("PDL launch,   %4u blocks: %.2f us per dependent kernel\n", blocks, ms * 1e3 / iters);
  }
  // host round trips
  unsigned *hp, *hmapped, *dmapped;
  CK(cudaHostAlloc(&hp, 64, cudaHostAllocDefault));
  CK(cudaHostAlloc(&hmapped, 64, cudaHostAllocMapped));
  CK(cudaHostGetDevicePointer(&dmapped, hmapped, 0));
  const int rt = 500;
  double t0 = now_us();
  for (int i = 0; i < rt; ++i) {
    tiny<<<1, 256, 0, s>>>(d, 256);
    CK(cudaMemcpyAsync(hp, d, 8, cudaMemcpyDeviceToHost, s));
    CK(cudaStreamSynchronize(s));
  }
  double t1 = now_us();
  printf("kernel + 8-byte D2H + cudaStreamSynchronize: %.2f us per round trip\n", (t1 - t0) / rt);
  t0 = now_us();
  for (int i = 0; i < rt; ++i) {
    tiny<<<1, 256, 0, s>>>(d, 256);
    CK(cudaStreamSynchronize(s));
  }
  t1 = now_us();
  printf("kernel + cudaStreamSynchronize: %.2f us per round trip\n", (t1 - t0) / rt);
  volatile unsigned* vh = hmapped;
  vh[0] = 0;
  t0 = now_us();
  for (int i = 1; i <= rt; ++i) {
    tiny<<<1, 256, 0, s>>>(d, 256);
    sizes_to_host<<<1, 32, 0, s>>>(d, dmapped, (unsigned)i);
    while (vh[0] != (unsigned)i) {
    }
  }
  t1 = now_us();
  printf("kernel + mapped-memory flag polled by the host: %.2f us per round trip\n", (t1 - t0) / rt);
  CK(cudaStreamSynchronize(s));
  printf("done\n");
  return 0;
}
