// FP64 global RED throughput on B200 by address pattern (S6, digestion):
//   pattern g: lanes in groups of g hit g consecutive doubles of one 32 B sector (g = 1: every lane its
//   own sector); elements/s over a buffer larger than L2 -> is the L2 atomic limit per element or per sector?
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/atomics_bench tools/atomics_bench.cu
#include <cstdio>
#include <cuda_runtime.h>

__global__ void red_kernel(double* __restrict__ buf, size_t nsec, int g, int iters, unsigned seed) {
  const int lane = threadIdx.x & 31;
  unsigned x = seed ^ (blockIdx.x * 9781u + threadIdx.x / 32 * 6271u);
  for (int it = 0; it < iters; ++it) {
    x = x * 1664525u + 1013904223u;
    unsigned grp = __shfl_sync(0xffffffffu, x, (lane / g) * g);  // same random sector for the group
    size_t sec = (size_t)(grp % (unsigned)nsec);
    double* p = buf + sec * 4 + (lane % g);
    atomicAdd(p, 1.0);
  }
}

int main() {
  const size_t n = (size_t)1 << 28;  // 2 GB of doubles
  double* buf;
  cudaMalloc(&buf, n * 8);
  cudaMemset(buf, 0, n * 8);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  int nsm = 0;
  cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0);
  for (int g : {1, 2, 4}) {
    const int iters = 2000, blocks = nsm * 8, threads = 256;
    red_kernel<<<blocks, threads>>>(buf, n / 4, g, 10, 1);
    cudaEventRecord(e0);
    red_kernel<<<blocks, threads>>>(buf, n / 4, g, iters, 7);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms = 0;
    cudaEventElapsedTime(&ms, e0, e1);
    const double el = (double)blocks * threads * iters;
    printf("{\"group\": %d, \"elements_per_s\": %.4g, \"sectors_per_s\": %.4g, \"ms\": %.2f}\n", g, el / (ms * 1e-3),
           el / g / (ms * 1e-3), ms);
  }
  return 0;
}
