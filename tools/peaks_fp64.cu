// FP64 peak microbenchmarks for B200 (sm_100a): DFMA loop, DMMA (mma.sync f64) loops,
// and DFMA+DMMA issued concurrently from different warps (does the tensor FP64 path share the DFMA pipe?).
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o peaks_fp64 peaks_fp64.cu
#include <cstdio>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("CUDA %s @%d\n", cudaGetErrorString(e), __LINE__); return 1; } } while (0)

constexpr int ITERS = 4096;

__global__ void dfma_loop(double* out, double s) {
  double a[16];
#pragma unroll
  for (int i = 0; i < 16; ++i) a[i] = threadIdx.x * 1e-3 + i;
  for (int it = 0; it < ITERS; ++it) {
#pragma unroll
    for (int i = 0; i < 16; ++i) a[i] = fma(a[i], s, 1e-7);
  }
  double r = 0;
#pragma unroll
  for (int i = 0; i < 16; ++i) r += a[i];
  if (r == 1.2345) out[threadIdx.x] = r;
}

__device__ __forceinline__ void dmma_16_8_4(double (&d)[4], double a0, double a1, double b0) {
  asm volatile("mma.sync.aligned.m16n8k4.row.col.f64.f64.f64.f64 {%0,%1,%2,%3}, {%4,%5}, {%6}, {%0,%1,%2,%3};\n"
               : "+d"(d[0]), "+d"(d[1]), "+d"(d[2]), "+d"(d[3]) : "d"(a0), "d"(a1), "d"(b0));
}
__device__ __forceinline__ void dmma_8_8_4(double (&d)[2], double a0, double b0) {
  asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};\n"
               : "+d"(d[0]), "+d"(d[1]) : "d"(a0), "d"(b0));
}

template <int NACC>
__global__ void dmma16_loop(double* out, double s) {
  double acc[NACC][4];
#pragma unroll
  for (int i = 0; i < NACC; ++i) for (int j = 0; j < 4; ++j) acc[i][j] = 0;
  double a0 = threadIdx.x * 1e-3, a1 = s, b0 = s * 0.5;
  for (int it = 0; it < ITERS; ++it) {
#pragma unroll
    for (int i = 0; i < NACC; ++i) dmma_16_8_4(acc[i], a0, a1, b0);
  }
  double r = 0;
#pragma unroll
  for (int i = 0; i < NACC; ++i) r += acc[i][0] + acc[i][1] + acc[i][2] + acc[i][3];
  if (r == 1.2345) out[threadIdx.x] = r;
}

template <int NACC>
__global__ void dmma8_loop(double* out, double s) {
  double acc[NACC][2];
#pragma unroll
  for (int i = 0; i < NACC; ++i) acc[i][0] = acc[i][1] = 0;
  double a0 = threadIdx.x * 1e-3, b0 = s * 0.5;
  for (int it = 0; it < ITERS; ++it) {
#pragma unroll
    for (int i = 0; i < NACC; ++i) dmma_8_8_4(acc[i], a0, b0);
  }
  double r = 0;
#pragma unroll
  for (int i = 0; i < NACC; ++i) r += acc[i][0] + acc[i][1];
  if (r == 1.2345) out[threadIdx.x] = r;
}

// half the warps do DMMA, half do DFMA
__global__ void mixed_loop(double* out, double s) {
  int w = threadIdx.x / 32;
  double r = 0;
  if (w & 1) {
    double acc[8][4];
    for (int i = 0; i < 8; ++i) for (int j = 0; j < 4; ++j) acc[i][j] = 0;
    double a0 = threadIdx.x * 1e-3, a1 = s, b0 = s * 0.5;
    for (int it = 0; it < ITERS; ++it) {
#pragma unroll
      for (int i = 0; i < 8; ++i) dmma_16_8_4(acc[i], a0, a1, b0);
    }
    for (int i = 0; i < 8; ++i) r += acc[i][0];
  } else {
    double a[16];
    for (int i = 0; i < 16; ++i) a[i] = threadIdx.x * 1e-3 + i;
    for (int it = 0; it < ITERS; ++it) {
#pragma unroll
      for (int i = 0; i < 16; ++i) a[i] = fma(a[i], s, 1e-7);
    }
    for (int i = 0; i < 16; ++i) r += a[i];
  }
  if (r == 1.2345) out[threadIdx.x] = r;
}

int main() {
  double* out; CK(cudaMalloc(&out, 1 << 20));
  int sms; CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0));
  int clk; CK(cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0));
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  auto timeit = [&](auto kern, int blocks, int threads, double flops_per_thread_iter, const char* name, double flop_total_override) {
    for (int w = 0; w < 3; ++w) kern<<<blocks, threads>>>(out, 0.999);
    cudaEventRecord(e0);
    const int REP = 10;
    for (int r = 0; r < REP; ++r) kern<<<blocks, threads>>>(out, 0.999);
    cudaEventRecord(e1); cudaEventSynchronize(e1);
    float ms; cudaEventElapsedTime(&ms, e0, e1);
    double flops = flop_total_override > 0 ? flop_total_override : (double)blocks * threads * flops_per_thread_iter * ITERS;
    double tf = flops * REP / (ms * 1e-3) / 1e12;
    printf("{\"kernel\": \"%s\", \"blocks\": %d, \"threads\": %d, \"tflops\": %.3f}\n", name, blocks, threads, tf);
    return tf;
  };
  printf("{\"sms\": %d, \"clock_khz\": %d}\n", sms, clk);
  for (int occ : {1, 2, 4, 8}) {
    timeit(dfma_loop, sms * occ, 256, 16 * 2.0, "dfma16x256", 0);
  }
  for (int occ : {1, 2, 4, 8}) {
    // per warp: NACC mma of 16*8*4*2 = 1024 flop per iter; per thread 1024/32 * NACC
    timeit(dmma16_loop<8>, sms * occ, 128, 8 * 1024.0 / 32, "dmma_m16n8k4_acc8x128", 0);
    timeit(dmma16_loop<4>, sms * occ, 256, 4 * 1024.0 / 32, "dmma_m16n8k4_acc4x256", 0);
    timeit(dmma8_loop<8>, sms * occ, 128, 8 * 512.0 / 32, "dmma_m8n8k4_acc8x128", 0);
  }
  for (int occ : {1, 2, 4}) {
    // half warps DMMA (8 acc => 8*1024/32 per thread), half DFMA (32 per thread)
    double f = (double)sms * occ * 128 * ITERS * (8 * 1024.0 / 32 + 32.0);
    timeit(mixed_loop, sms * occ, 256, 0, "mixed_dmma_dfma_256", f);
  }
  return 0;
}
