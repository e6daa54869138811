// Microbenchmark of the integrator's per-evaluation loop shapes on sm_100a (development tool,
// DESIGN sec. 7): how close to the FP64 pipe can the 27-node x 3-level x 3-component
// contraction run at 8 one-warp CTAs per SM (the register-bound residency of k_integrate)?
//   V0  contraction only: deltas from registers (no loads, no geometry)
//   V1  + per-node geometry record (dx, dy, w, cell) and node record (w0, w1, w2, wk, wg) read
//       from shared memory, cell test (the "phase C" of a two-phase round)
//   V2  V1 + a refill of the 27-node stencil (27 x 256-bit loads, L1-resident) on 1/8 of the
//       lane-evaluations (divergent, as in the bend)
//   V3  V2 with the refill on 1/32
// Prints cycles per warp-evaluation per scheduler and the FP64 pipe fraction implied by the
// SASS DFMA/DMUL/DADD count of the loop (2 cycles per warp FP64 instruction per scheduler).
#include <cstdio>
#include <cuda_runtime.h>

__device__ __forceinline__ void ldg_node(const double* p, double& a, double& b, double& c) {
  double d;
  asm volatile("ld.global.nc.v4.f64 {%0,%1,%2,%3}, [%4];" : "=d"(a), "=d"(b), "=d"(c), "=d"(d) : "l"(p));
}

struct NodeRec { double r, cu, cv, w0, w1, w2, wk, wg; };

template <int V>
__global__ void __launch_bounds__(32) kloop(const double* __restrict__ in, double* out,
                                             long long* cyc, int iters,
                                             const double* __restrict__ ring, int refill_mod) {
  __shared__ double2 sdxy[16][32];
  __shared__ double sw[16][32];
  __shared__ int scell[16][32];
  __shared__ NodeRec snode[16];
  const int lane = threadIdx.x;
  for (int n = 0; n < 16; ++n) {
    sdxy[n][lane] = make_double2(lane * 1e-3 + n * 1e-2 - 0.2, 0.25 - lane * 1e-3);
    sw[n][lane] = 0.01 * (n + 1);
    scell[n][lane] = 200 + lane + (n / 4);
    if (lane == 0) snode[n] = NodeRec{1.0, 2.0, 3.0, 0.2 + n * 1e-3, 0.7, 0.1, 0.05, 0.03};
  }
  __syncwarp();
  double st[3][9][3];
#pragma unroll
  for (int l = 0; l < 3; ++l)
#pragma unroll
    for (int i = 0; i < 9; ++i)
#pragma unroll
      for (int c = 0; c < 3; ++c) st[l][i][c] = in[(l * 27 + i * 3 + c + lane) & 127];
  double k0 = 0, k1 = 0, k2 = 0, g0 = 0, g1 = 0, g2 = 0;
  double rdx = lane * 1e-3, rdy = 0.25 - lane * 1e-3;
  int ccell = -1;
  const int PX = 70;
  long long t0 = clock64();
  for (int it = 0; it < iters; ++it) {
#pragma unroll 1
    for (int n = 0; n < 15; ++n) {
      double dx, dy, w, w0, w1, w2, wk, wg;
      if (V == 0) {
        dx = rdx; dy = rdy; w = 0.01; w0 = 0.2; w1 = 0.7; w2 = 0.1; wk = 0.05; wg = 0.03;
        rdx = fma(rdx, 0.999, 1e-4);
        rdy = fma(rdy, 0.999, -1e-4);
      } else {
        const double2 d = sdxy[n][lane];
        dx = d.x; dy = d.y; w = sw[n][lane];
        const int cell = scell[n][lane] + ((V >= 2 && ((it * 15 + n + lane * 7) % refill_mod) == 0) ? it : 0);
        if (V >= 2 && cell != ccell) {
          ccell = cell;
          const double* g = ring + 4 * (size_t)(cell % 4000);
#pragma unroll
          for (int l = 0; l < 3; ++l)
#pragma unroll
            for (int b = 0; b < 3; ++b)
#pragma unroll
              for (int a = 0; a < 3; ++a)
                ldg_node(g + 4 * (l * 4900 + b * PX + a), st[l][3 * b + a][0], st[l][3 * b + a][1],
                         st[l][3 * b + a][2]);
        }
        const NodeRec& nd = snode[n];
        w0 = nd.w0; w1 = nd.w1; w2 = nd.w2; wk = nd.wk; wg = nd.wg;
      }
      const double ax = 0.5 - dx, bx = 0.5 + dx, ay = 0.5 - dy, by = 0.5 + dy;
      const double wx[3] = {ax * ax, fma(-2.0 * dx, dx, 1.5), bx * bx};
      const double wy[3] = {ay * ay, fma(-2.0 * dy, dy, 1.5), by * by};
      double s[3][3];
      const double w00 = wx[0] * wy[0];
#pragma unroll
      for (int l = 0; l < 3; ++l)
#pragma unroll
        for (int c = 0; c < 3; ++c) s[l][c] = w00 * st[l][0][c];
#pragma unroll
      for (int i = 1; i < 9; ++i) {
        const double ww = wx[i % 3] * wy[i / 3];
#pragma unroll
        for (int l = 0; l < 3; ++l)
#pragma unroll
          for (int c = 0; c < 3; ++c) s[l][c] = fma(ww, st[l][i][c], s[l][c]);
      }
      const double f0 = w0 * s[0][0] + w1 * s[1][0] + w2 * s[2][0];
      const double f1 = w0 * s[0][1] + w1 * s[1][1] + w2 * s[2][1];
      const double f2 = w0 * s[0][2] + w1 * s[1][2] + w2 * s[2][2];
      const double wkk = 0.25 * w * wk;
      k0 += wkk * f0; k1 += wkk * f1; k2 += wkk * f2;
      if (n & 1) {
        const double wgg = 0.25 * w * wg;
        g0 += wgg * f0; g1 += wgg * f1; g2 += wgg * f2;
      }
    }
  }
  long long t1 = clock64();
  out[blockIdx.x * 32 + lane] = k0 + k1 + k2 + g0 + g1 + g2;
  if (lane == 0) cyc[blockIdx.x] = t1 - t0;
}

int main() {
  double *in, *out, *ring;
  long long* cyc;
  cudaMalloc(&in, 128 * 8);
  cudaMalloc(&out, 1 << 20);
  cudaMalloc(&cyc, 1 << 16);
  cudaMemset(in, 0, 128 * 8);
  const size_t rb = (size_t)4 * 4900 * 4 * 8;
  cudaMalloc(&ring, rb);
  cudaMemset(ring, 0, rb);
  int clk;
  cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
  const int iters = 2048;
  for (int v = 0; v < 4; ++v) {
    for (int ctas_per_sm = 4; ctas_per_sm <= 12; ctas_per_sm += 4) {
      const int blocks = 148 * ctas_per_sm;
      const int mod = v == 2 ? 8 : 32;
      auto launch = [&]() {
        if (v == 0) kloop<0><<<blocks, 32>>>(in, out, cyc, iters, ring, mod);
        else if (v == 1) kloop<1><<<blocks, 32>>>(in, out, cyc, iters, ring, mod);
        else kloop<2><<<blocks, 32>>>(in, out, cyc, iters, ring, mod);
      };
      launch();
      cudaDeviceSynchronize();
      cudaEvent_t e0, e1;
      cudaEventCreate(&e0);
      cudaEventCreate(&e1);
      cudaEventRecord(e0);
      launch();
      cudaEventRecord(e1);
      cudaEventSynchronize(e1);
      float ms;
      cudaEventElapsedTime(&ms, e0, e1);
      const double warp_evals_per_smsp = (double)ctas_per_sm / 4.0 * iters * 15.0;
      const double cycles = ms * 1e-3 * clk * 1e3;
      printf("{\"variant\": %d, \"warps_per_sm\": %d, \"ms\": %.3f, \"cycles_per_warp_eval_per_smsp\": %.1f}\n",
             v, ctas_per_sm, ms, cycles / warp_evals_per_smsp);
    }
  }
  cudaError_t e = cudaGetLastError();
  if (e) printf("err %s\n", cudaGetErrorString(e));
  return 0;
}
