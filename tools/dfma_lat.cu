// DFMA dependent-chain latency and per-SMSP throughput vs independent chains per warp and
// warps per scheduler (sm_100a).  One CTA of 4*W warps on one SM (W warps per SMSP).
#include <cstdio>
#include <cuda_runtime.h>
template <int C>
__global__ void chain(double* out, long long* cyc, int iters) {
  double x[C];
#pragma unroll
  for (int i = 0; i < C; ++i) x[i] = threadIdx.x * 1e-3 + i;
  __syncthreads();
  long long t0 = clock64();
  for (int it = 0; it < iters; ++it)
#pragma unroll
    for (int i = 0; i < C; ++i) x[i] = fma(x[i], 0.999999, 1e-7);
  __syncthreads();
  long long t1 = clock64();
  double s = 0;
#pragma unroll
  for (int i = 0; i < C; ++i) s += x[i];
  if (s == 1234.5) out[0] = s;
  if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
}
template <int C>
void run(int w, double* out, long long* cyc) {
  int iters = 2048;
  chain<C><<<1, 128 * w>>>(out, cyc, iters);
  cudaDeviceSynchronize();
  long long h;
  cudaMemcpy(&h, cyc, 8, cudaMemcpyDeviceToHost);
  // per SMSP: w warps x C chains x iters DFMA warp-instructions
  double per = (double)h / ((double)iters * C * w);
  printf("{\"chains\": %d, \"warps_per_smsp\": %d, \"smsp_cycles_per_warp_dfma\": %.2f}\n", C, w, per);
}
int main() {
  double* out; long long* cyc;
  cudaMalloc(&out, 8); cudaMalloc(&cyc, 8 * 16);
  for (int w = 1; w <= 4; ++w) {
    run<1>(w, out, cyc); run<2>(w, out, cyc); run<4>(w, out, cyc); run<6>(w, out, cyc);
    run<9>(w, out, cyc); run<12>(w, out, cyc); run<16>(w, out, cyc);
  }
  return 0;
}
