// DFMA dependent-chain latency and per-SMSP throughput vs chains/warps (sm_100a).
#include <cstdio>
#include <cuda_runtime.h>
template <int C>
__global__ void chain(double* out, long long* cyc, int iters) {
  double x[C];
#pragma unroll
  for (int i = 0; i < C; ++i) x[i] = threadIdx.x * 1e-3 + i;
  long long t0 = clock64();
  for (int it = 0; it < iters; ++it)
#pragma unroll
    for (int i = 0; i < C; ++i) x[i] = fma(x[i], 0.999999, 1e-7);
  long long t1 = clock64();
  double s = 0;
#pragma unroll
  for (int i = 0; i < C; ++i) s += x[i];
  if (s == 1234.5) out[0] = s;
  if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
}
template <int C>
void run(int warps, double* out, long long* cyc) {
  int iters = 4096;
  chain<C><<<1, 32 * warps>>>(out, cyc, iters);
  cudaDeviceSynchronize();
  long long h;
  cudaMemcpy(&h, cyc, 8, cudaMemcpyDeviceToHost);
  double per = (double)h / (iters * C);
  printf("{\"chains\": %d, \"warps_in_block\": %d, \"cycles_per_dfma_per_warp\": %.2f}\n", C, warps, per);
}
int main() {
  double* out; long long* cyc;
  cudaMalloc(&out, 8); cudaMalloc(&cyc, 8 * 16);
  run<1>(1, out, cyc); run<2>(1, out, cyc); run<4>(1, out, cyc); run<8>(1, out, cyc);
  run<1>(4, out, cyc); run<4>(4, out, cyc); run<8>(4, out, cyc);
  run<1>(8, out, cyc); run<4>(8, out, cyc); run<8>(8, out, cyc);
  run<1>(16, out, cyc); run<4>(16, out, cyc);
  return 0;
}
