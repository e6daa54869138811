// FP64 (DFMA) peak microbenchmark for the roofline denominator.
// Each thread runs 8 independent DFMA chains; grid = 148 SMs x 8 CTAs x 256 threads.
#include <cstdio>
#include <cuda_runtime.h>
__global__ void dfma_loop(double* out, int iters, double a, double b) {
  double x0 = threadIdx.x * 1e-3, x1 = x0 + 1, x2 = x0 + 2, x3 = x0 + 3,
         x4 = x0 + 4, x5 = x0 + 5, x6 = x0 + 6, x7 = x0 + 7;
  for (int i = 0; i < iters; ++i) {
#pragma unroll
    for (int u = 0; u < 16; ++u) {
      x0 = fma(x0, a, b); x1 = fma(x1, a, b); x2 = fma(x2, a, b); x3 = fma(x3, a, b);
      x4 = fma(x4, a, b); x5 = fma(x5, a, b); x6 = fma(x6, a, b); x7 = fma(x7, a, b);
    }
  }
  double s = x0 + x1 + x2 + x3 + x4 + x5 + x6 + x7;
  if (s == 12345.678) out[0] = s;
}
int main() {
  int dev = 0, sms = 0, clk = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, dev);
  double* out; cudaMalloc(&out, 8);
  int blocks = sms * 4, threads = 256, iters = 4096;  // 32 warps / SM
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  for (int w = 0; w < 3; ++w) dfma_loop<<<blocks, threads>>>(out, iters, 0.999999, 1e-7);
  float best = 1e30f;
  for (int r = 0; r < 10; ++r) {
    cudaEventRecord(e0);
    dfma_loop<<<blocks, threads>>>(out, iters, 0.999999, 1e-7);
    cudaEventRecord(e1); cudaEventSynchronize(e1);
    float ms; cudaEventElapsedTime(&ms, e0, e1); if (ms < best) best = ms;
  }
  double flops = 2.0 * 8 * 16 * (double)iters * blocks * threads;
  printf("{\"sms\": %d, \"clock_khz_attr\": %d, \"fp64_tflops_burst\": %.3f, \"ms\": %.3f}\n",
         sms, clk, flops / (best * 1e-3) / 1e12, best);
  // sustained: back to back for ~3 s
  cudaEventRecord(e0); int n = 0; float ms = 0;
  while (ms < 3000.f) {
    for (int r = 0; r < 20; ++r) dfma_loop<<<blocks, threads>>>(out, iters, 0.999999, 1e-7);
    n += 20; cudaEventRecord(e1); cudaEventSynchronize(e1); cudaEventElapsedTime(&ms, e0, e1);
  }
  printf("{\"fp64_tflops_sustained\": %.3f, \"launches\": %d}\n", flops * n / (ms * 1e-3) / 1e12, n);
  return 0;
}
