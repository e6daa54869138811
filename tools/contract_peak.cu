// Throughput of the integrator's contraction alone (sm_100a): 81 cached doubles in registers,
// per point 2x3 TSC weights, 9 products, 81-term 9-chain DFMA contraction, time combination,
// K accumulation -- no geometry, no loads.  Reports cycles per point per warp and the DFMA
// rate, at 1 and 2 warps per scheduler.
#include <cstdio>
#include <cuda_runtime.h>
__constant__ double c_sinp[6] = {1.58969099521155010221e-10, -2.50507602534068634195e-08,
                                 2.75573137070700676789e-06, -1.98412698298579493134e-04,
                                 8.33333333332248946124e-03, -1.66666666666666324348e-01};
__constant__ double c_cosp[6] = {-1.13596475577881948265e-11, 2.08757232129817482790e-09,
                                 -2.75573143513906633035e-07, 2.48015872894767294178e-05,
                                 -1.38888888888741095749e-03, 4.16666666666666019037e-02};
__device__ __forceinline__ void sincos_b(double x, double* s, double* c) {
  const double k = rint(x * 0.63661977236758134308);
  double r = fma(-k, 1.5707963267948965580, x);
  r = fma(-k, 6.1232339957367658e-17, r);
  const double z = r * r;
  double ps = fma(z, c_sinp[0], c_sinp[1]);
  ps = fma(z, ps, c_sinp[2]); ps = fma(z, ps, c_sinp[3]); ps = fma(z, ps, c_sinp[4]); ps = fma(z, ps, c_sinp[5]);
  const double sr = fma(r * z, ps, r);
  double pc = fma(z, c_cosp[0], c_cosp[1]);
  pc = fma(z, pc, c_cosp[2]); pc = fma(z, pc, c_cosp[3]); pc = fma(z, pc, c_cosp[4]); pc = fma(z, pc, c_cosp[5]);
  const double cr = fma(z * z, pc, fma(-0.5, z, 1.0));
  const int q = (int)k & 3;
  const double ss = (q & 1) ? cr : sr, cc = (q & 1) ? sr : cr;
  *s = (q & 2) ? -ss : ss;
  *c = ((q + 1) & 2) ? -cc : cc;
}
__device__ __forceinline__ void ldg_node(const double* p, double& a, double& b, double& c) {
  double d;
  asm volatile("ld.global.nc.v4.f64 {%0,%1,%2,%3}, [%4];" : "=d"(a), "=d"(b), "=d"(c), "=d"(d) : "l"(p));
}
template <bool GEO, int REFILL>
__global__ void __launch_bounds__(32) kcon(const double* __restrict__ in, double* out, long long* cyc, int iters,
                                           const double* __restrict__ ring) {
  double st[3][9][3];
#pragma unroll
  for (int l = 0; l < 3; ++l)
#pragma unroll
    for (int i = 0; i < 9; ++i)
#pragma unroll
      for (int c = 0; c < 3; ++c) st[l][i][c] = in[(l * 27 + i * 3 + c + threadIdx.x) & 127];
  double k0 = 0, k1 = 0, k2 = 0;
  double dx = threadIdx.x * 1e-3, dy = 0.25 - threadIdx.x * 1e-3;
  const double w0 = 0.2, w1 = 0.7, w2 = 0.1;
  long long t0 = clock64();
  const int PX = 70;
  int cell = 200 + 3 * (int)threadIdx.x + 4900 * (int)(blockIdx.x % 40);
  for (int it = 0; it < iters; ++it) {
    if (REFILL && ((it * 7 + threadIdx.x * 3) % REFILL) == 0) {
      cell += 1 + ((it >> 4) & 1) * (PX - 1);  // walk along a strip
      if (cell > 4900 * 100) cell -= 4900 * 90;
      const double* g = ring + 4 * (size_t)cell;
#pragma unroll
      for (int l = 0; l < 3; ++l)
#pragma unroll
        for (int b = 0; b < 3; ++b)
#pragma unroll
          for (int a = 0; a < 3; ++a)
            ldg_node(g + 4 * (l * 4900 + b * PX + a), st[l][3 * b + a][0], st[l][3 * b + a][1], st[l][3 * b + a][2]);
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
    k0 += 0.3 * f0; k1 += 0.3 * f1; k2 += 0.3 * f2;
    if (GEO) {  // next point: arc angle -> sincos -> cell coordinate -> floor -> fraction
      double sn, cs;
      sincos_b(fma((double)(it & 63), 1e-3, 0.1 * threadIdx.x), &sn, &cs);
      const double tx = fma(6000.0, cs, 12.3 + dx), ty = fma(6000.0, sn, 7.7 + dy);
      const double fx = floor(tx + 0.5), fy = floor(ty + 0.5);
      dx = tx - fx; dy = ty - fy;
    } else {
      dx = fma(dx, 0.999, 1e-4); dy = fma(dy, 0.999, -1e-4);
    }
  }
  long long t1 = clock64();
  out[blockIdx.x * 32 + threadIdx.x] = k0 + k1 + k2;
  if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
}
int main() {
  double *in, *out; long long* cyc;
  cudaMalloc(&in, 128 * 8); cudaMalloc(&out, 65536 * 8); cudaMalloc(&cyc, 4096 * 8);
  cudaMemset(in, 0, 128 * 8);
  double* ring; cudaMalloc(&ring, (size_t)4 * 4900 * 102 * 8); cudaMemset(ring, 0, (size_t)4 * 4900 * 102 * 8);
  const int iters = 4096;
  for (int wps = 1; wps <= 2; ++wps) {
    // 4*wps one-warp CTAs on one SM: force co-residency by launching exactly that many blocks
    // on a 1-SM slice is not possible; launch 148*4*wps blocks (all SMs) and take the max.
    int blocks = 148 * 4 * wps;
    for (int geo = 0; geo < 4; ++geo) {
    auto launch = [&]() {
      if (geo == 0) kcon<false, 0><<<blocks, 32>>>(in, out, cyc, iters, ring);
      else if (geo == 1) kcon<true, 0><<<blocks, 32>>>(in, out, cyc, iters, ring);
      else if (geo == 2) kcon<true, 3><<<blocks, 32>>>(in, out, cyc, iters, ring);
      else kcon<true, 10><<<blocks, 32>>>(in, out, cyc, iters, ring);
    };
    launch();
    cudaDeviceSynchronize();
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
    cudaEventRecord(e0);
    launch();
    cudaEventRecord(e1); cudaEventSynchronize(e1);
    float ms; cudaEventElapsedTime(&ms, e0, e1);
    int clk; cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
    double pts = (double)blocks * iters;  // warp-points
    printf("{\"variant(0 contr,1 +geo,2 +refill/3,3 +refill/10)\": %d, \"warps_per_smsp\": %d, \"event_ms\": %.3f, \"smsp_cycles_per_warp_point_wall\": %.1f}\n",
           geo, wps, ms, ms * 1e-3 * clk * 1e3 * 148 * 4 / pts);
    }
  }
  cudaError_t e = cudaGetLastError();
  if (e) printf("err %s\n", cudaGetErrorString(e));
  return 0;
}
