#include <cstdlib>
// Do DMMA (tensor) and DFMA (FP64 pipe) run concurrently on sm_100a?  Mixed-loop throughput.
#include <cstdio>
#include <cuda_runtime.h>
template <int NM, int NF>
__global__ void mix_loop(double* out, int iters) {
  double a = threadIdx.x * 1e-3, b = 1.0 + threadIdx.x * 1e-4;
  double c[8][2];
  double x[8];
#pragma unroll
  for (int i = 0; i < 8; ++i) { c[i][0] = c[i][1] = 0.0; x[i] = i * 1e-3; }
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int i = 0; i < NM; ++i)
      asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};"
                   : "+d"(c[i][0]), "+d"(c[i][1]) : "d"(a), "d"(b));
#pragma unroll
    for (int r = 0; r < NF; ++r)
#pragma unroll
      for (int i = 0; i < 8; ++i) x[i] = fma(x[i], 0.999999, 1e-7);
  }
  double s = 0;
#pragma unroll
  for (int i = 0; i < 8; ++i) s += c[i][0] + c[i][1] + x[i];
  if (s == 1234.5) out[0] = s;
}
template <int NM, int NF>
void run(int sms, double* out) {
  int iters = 1024, blocks = sms * 4, threads = 256;
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  mix_loop<NM, NF><<<blocks, threads>>>(out, iters);
  cudaEventRecord(e0);
  for (int r = 0; r < 5; ++r) mix_loop<NM, NF><<<blocks, threads>>>(out, iters);
  cudaEventRecord(e1); cudaEventSynchronize(e1);
  float ms; cudaEventElapsedTime(&ms, e0, e1);
  double warps = (double)blocks * threads / 32;
  double mma_fl = 5.0 * iters * warps * NM * 512.0;       // 256 FMA per DMMA
  double fma_fl = 5.0 * iters * blocks * threads * NF * 8 * 2.0;
  printf("{\"dmma_per_iter\": %d, \"dfma_rounds\": %d, \"ms\": %.3f, \"dmma_tf\": %.2f, \"dfma_tf\": %.2f, \"total_tf\": %.2f}\n",
         NM, NF, ms, mma_fl / (ms * 1e-3) / 1e12, fma_fl / (ms * 1e-3) / 1e12,
         (mma_fl + fma_fl) / (ms * 1e-3) / 1e12);
}
int main(int argc, char** argv) {
  int sms = 0; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  double* out; cudaMalloc(&out, 8);
  const int reps = argc > 1 ? atoi(argv[1]) : 1;  // repeat the pure DFMA / DMMA runs (clock logs)
  for (int r = 1; r < reps; ++r) { run<0, 8>(sms, out); run<8, 0>(sms, out); }
  run<8, 0>(sms, out);
  run<0, 8>(sms, out);
  run<8, 8>(sms, out);
  run<4, 16>(sms, out);
  run<8, 16>(sms, out);
  return 0;
}
