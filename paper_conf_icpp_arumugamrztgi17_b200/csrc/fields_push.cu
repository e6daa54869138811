// fields_push.cu -- steps 3 and 4 of the paper's loop (P:58 self-forces from the potentials,
// P:60 leap-frog Lorentz push).  Both are O(N_x N_y) / O(N) streaming kernels bound by HBM;
// one thread per mesh node / particle, coalesced SoA access.
#include <algorithm>

#include "rp_internal.cuh"

namespace {

// second-order derivative along u (dir 0) or v (dir 1); one-sided at the edges (R-15)
__device__ __forceinline__ double dd(const double* __restrict__ f, int nx, int ny, int ix, int iy,
                                     int dir, double h) {
  int n = dir == 0 ? nx : ny, i = dir == 0 ? ix : iy;
  size_t s = dir == 0 ? 1 : (size_t)nx;
  const double* p = f + (size_t)iy * nx + ix;
  if (i == 0) return (-3.0 * p[0] + 4.0 * p[s] - p[2 * s]) / (2.0 * h);
  if (i == n - 1) return (3.0 * p[0] - 4.0 * p[-(ptrdiff_t)s] + p[-2 * (ptrdiff_t)s]) / (2.0 * h);
  return (p[s] - p[-(ptrdiff_t)s]) / (2.0 * h);
}

// order-m backward-difference weights (R-15b), units of 1/dt: f'(t_k) ~ sum_j BD[m][j] f(t_{k-j})
__constant__ double c_bd[5][5] = {{0, 0, 0, 0, 0},
                                  {1.0, -1.0, 0, 0, 0},
                                  {1.5, -2.0, 0.5, 0, 0},
                                  {11.0 / 6.0, -3.0, 1.5, -1.0 / 3.0, 0},
                                  {25.0 / 12.0, -4.0, 3.0, -4.0 / 3.0, 0.25}};

struct FieldFrames {
  rp_frame f[5];  // levels k, k-1, ..., k-m
};

// E = -grad phi - (1/c) dA/dt, B_z = d_x A_y - d_y A_x on mesh k.  The mesh moves with
// its frame: dA/dt|lab = (1/dt) sum_j BD[m][j] A_{k-j}(node) - (V . grad) A_k with the node
// velocity V = (1/dt) sum_j BD[m][j] P_{k-j}(node) -- consistent order-m backward differences
// at t_k (R-15b); aprev [m][2][npts] holds A of steps k-1 .. k-m.
__global__ void k_fields(int nx, int ny, double hx, double hy, double c, double dt,
                         FieldFrames F, int m, const double* __restrict__ phi,
                         const double* __restrict__ ax, const double* __restrict__ ay,
                         const double* __restrict__ aprev, double* __restrict__ ex,
                         double* __restrict__ ey, double* __restrict__ bz) {
  int id = blockIdx.x * blockDim.x + threadIdx.x;
  const int npts = nx * ny;
  if (id >= npts) return;
  int ix = id % nx, iy = id / nx;
  const rp_frame& Fk = F.f[0];
  double cs = Fk.cos_psi, sn = Fk.sin_psi;
  double pu = dd(phi, nx, ny, ix, iy, 0, hx), pv = dd(phi, nx, ny, ix, iy, 1, hy);
  double xu = dd(ax, nx, ny, ix, iy, 0, hx), xv = dd(ax, nx, ny, ix, iy, 1, hy);
  double yu = dd(ay, nx, ny, ix, iy, 0, hx), yv = dd(ay, nx, ny, ix, iy, 1, hy);
  double phx = cs * pu - sn * pv, phy = sn * pu + cs * pv;
  double axx = cs * xu - sn * xv, axy = sn * xu + cs * xv;  // d_x A_x, d_y A_x
  double ayx = cs * yu - sn * yv, ayy = sn * yu + cs * yv;  // d_x A_y, d_y A_y
  double dax = 0.0, day = 0.0;
  if (m >= 1) {
    const double u = ix * hx, v = iy * hy;
    double vx = 0.0, vy = 0.0, nax = c_bd[m][0] * ax[id], nay = c_bd[m][0] * ay[id];
    for (int j = 0; j <= m; ++j) {
      const rp_frame& Fj = F.f[j];
      const double px = Fj.ox + u * Fj.cos_psi - v * Fj.sin_psi;
      const double py = Fj.oy + u * Fj.sin_psi + v * Fj.cos_psi;
      vx += c_bd[m][j] * px;
      vy += c_bd[m][j] * py;
      if (j >= 1) {
        nax += c_bd[m][j] * aprev[(size_t)(j - 1) * 2 * npts + id];
        nay += c_bd[m][j] * aprev[(size_t)(j - 1) * 2 * npts + npts + id];
      }
    }
    dax = (nax - (vx * axx + vy * axy)) / dt;
    day = (nay - (vx * ayx + vy * ayy)) / dt;
  }
  ex[id] = -phx - dax / c;
  ey[id] = -phy - day / c;
  bz[id] = ayx - axy;
}

__device__ __forceinline__ void tsc(double d, double& wm, double& w0, double& wp) {
  double a = 0.5 - d, b = 0.5 + d;
  wm = 0.5 * (a * a);
  w0 = 0.75 - d * d;
  wp = 0.5 * (b * b);
}

// TSC gather of (E_x, E_y, B_z) at lab point (X, Y) on frame F, with the deposition's weights
// (R-15); nodes outside the grid contribute 0
__device__ __forceinline__ void gather_eb(double X, double Y, const rp_frame& F, int nx, int ny,
                                          double inv_hx, double inv_hy,
                                          const double* __restrict__ ex,
                                          const double* __restrict__ ey,
                                          const double* __restrict__ bz, double& Ex, double& Ey,
                                          double& Bz) {
  double dx = X - F.ox, dy = Y - F.oy;
  double u = F.cos_psi * dx + F.sin_psi * dy;
  double v = F.cos_psi * dy - F.sin_psi * dx;
  double tx = u * inv_hx, ty = v * inv_hy;
  double fx = floor(tx + 0.5), fy = floor(ty + 0.5);
  Ex = 0.0; Ey = 0.0; Bz = 0.0;
  if (fx >= -2.0 && fx <= nx + 1.0 && fy >= -2.0 && fy <= ny + 1.0) {
    double wx[3], wy[3];
    tsc(tx - fx, wx[0], wx[1], wx[2]);
    tsc(ty - fy, wy[0], wy[1], wy[2]);
    int ix = (int)fx, iy = (int)fy;
#pragma unroll
    for (int b = 0; b < 3; ++b) {
      int yy = iy + b - 1;
      if (yy < 0 || yy >= ny) continue;
#pragma unroll
      for (int a = 0; a < 3; ++a) {
        int xx = ix + a - 1;
        if (xx < 0 || xx >= nx) continue;
        size_t id = (size_t)yy * nx + xx;
        double w = wx[a] * wy[b];
        Ex += w * __ldg(ex + id);
        Ey += w * __ldg(ey + id);
        Bz += w * __ldg(bz + id);
      }
    }
  }
}

// Lorentz force per unit charge on each particle, F = E + beta x (B_z + B_ext) z-hat, from the
// push's gather: the particle-level force of the paper's validation
__global__ void k_forces(int64_t n, const double* __restrict__ x, const double* __restrict__ y,
                         const double* __restrict__ ux, const double* __restrict__ uy, rp_frame F,
                         int nx, int ny, double inv_hx, double inv_hy, double bz_ext,
                         const double* __restrict__ ex, const double* __restrict__ ey,
                         const double* __restrict__ bz, double* __restrict__ fx,
                         double* __restrict__ fy) {
  int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (i >= n) return;
  double Ex, Ey, Bz;
  gather_eb(x[i], y[i], F, nx, ny, inv_hx, inv_hy, ex, ey, bz, Ex, Ey, Bz);
  Bz += bz_ext;
  const double a = ux[i], b = uy[i];
  const double g = sqrt(1.0 + a * a + b * b);
  fx[i] = Ex + (b / g) * Bz;
  fy[i] = Ey - (a / g) * Bz;
}

// time-centred momenta for the current (R-27): u advanced by frac * dt in the uniform external
// B_z (the push's Boris rotation with E = 0)
__global__ void k_kick_external(int64_t n, const double* __restrict__ ux,
                                const double* __restrict__ uy, double h, double bz_ext,
                                double* __restrict__ ox, double* __restrict__ oy) {
  int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (i >= n) return;
  const double a = ux[i], b = uy[i];
  const double gm = sqrt(1.0 + a * a + b * b);
  const double t = h * bz_ext / gm;
  const double sr = 2.0 * t / (1.0 + t * t);
  const double upx = a + b * t, upy = b - a * t;
  ox[i] = a + upy * sr;
  oy[i] = b - upx * sr;
}

__global__ void k_push(int64_t n, double* __restrict__ x, double* __restrict__ y,
                       double* __restrict__ ux, double* __restrict__ uy, rp_frame F, int nx,
                       int ny, double inv_hx, double inv_hy, double c, double dt, double qmc,
                       double bz_ext, const double* __restrict__ ex,
                       const double* __restrict__ ey, const double* __restrict__ bz) {
  int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (i >= n) return;
  double X = x[i], Y = y[i];
  double Ex, Ey, Bz;
  gather_eb(X, Y, F, nx, ny, inv_hx, inv_hy, ex, ey, bz, Ex, Ey, Bz);
  Bz += bz_ext;
  double h = 0.5 * qmc * dt;
  double umx = ux[i] + h * Ex, umy = uy[i] + h * Ey;
  double gm = sqrt(1.0 + umx * umx + umy * umy);
  double t = h * Bz / gm;
  double s = 2.0 * t / (1.0 + t * t);
  double upx = umx + umy * t, upy = umy - umx * t;
  double ppx = umx + upy * s, ppy = umy - upx * s;
  double nux = ppx + h * Ex, nuy = ppy + h * Ey;
  double g = sqrt(1.0 + nux * nux + nuy * nuy);
  ux[i] = nux;
  uy[i] = nuy;
  x[i] = X + c * dt * nux / g;
  y[i] = Y + c * dt * nuy / g;
}

}  // namespace

int rp_fields_impl(rp_ctx* ctx, const double* phi, const double* ax, const double* ay,
                   const double* a_prev, int n_prev, double* ex, double* ey, double* bz) {
  const rp_config& c = ctx->cfg;
  if (ctx->k < 0) return rp_fail(ctx, RP_ESTATE, "fields before the first deposit");
  if (!phi || !ax || !ay || !ex || !ey || !bz) return rp_fail(ctx, RP_EINVAL, "fields: null array");
  if (n_prev < 0 || n_prev > 4 || (n_prev > 0 && !a_prev))
    return rp_fail(ctx, RP_EINVAL, "fields: n_prev must be 0..4 with a_prev given");
  // order: the previous potentials given, limited by the frames the ring holds (levels down to
  // -n_pre exist; at most H - 1 back)
  int m = n_prev;
  m = std::min(m, ctx->H - 1);
  m = std::min(m, ctx->k + ctx->n_pre);
  m = std::max(m, 0);
  FieldFrames F;
  for (int j = 0; j <= 4; ++j) F.f[j] = ctx->fh[slot_of(ctx->k - (j <= m ? j : 0), ctx->H)];
  int npts = c.nx * c.ny;
  ProfScope ps(ctx, PK_FIELDS);
  k_fields<<<(npts + 255) / 256, 256, 0, ctx->stream>>>(c.nx, c.ny, c.hx, c.hy, c.c, c.dt, F, m,
                                                         phi, ax, ay, a_prev, ex, ey, bz);
  RP_CHECK_LAUNCH();
  return RP_OK;
}

int rp_push_impl(rp_ctx* ctx, double* x, double* y, double* ux, double* uy, int64_t n, double qmc,
                 double bz_ext, const double* ex, const double* ey, const double* bz) {
  const rp_config& c = ctx->cfg;
  if (ctx->k < 0) return rp_fail(ctx, RP_ESTATE, "push before the first deposit");
  if (n < 0) return rp_fail(ctx, RP_EINVAL, "push: n < 0");
  if (n == 0) return RP_OK;
  if (!x || !y || !ux || !uy || !ex || !ey || !bz) return rp_fail(ctx, RP_EINVAL, "push: null array");
  rp_frame Fk = ctx->fh[slot_of(ctx->k, ctx->H)];
  ProfScope ps(ctx, PK_PUSH);
  k_push<<<(unsigned)((n + 255) / 256), 256, 0, ctx->stream>>>(n, x, y, ux, uy, Fk, c.nx, c.ny,
                                                                1.0 / c.hx, 1.0 / c.hy, c.c, c.dt,
                                                                qmc, bz_ext, ex, ey, bz);
  RP_CHECK_LAUNCH();
  return RP_OK;
}

int rp_forces_impl(rp_ctx* ctx, const double* x, const double* y, const double* ux,
                   const double* uy, int64_t n, double bz_ext, const double* ex, const double* ey,
                   const double* bz, double* fx, double* fy) {
  const rp_config& c = ctx->cfg;
  if (ctx->k < 0) return rp_fail(ctx, RP_ESTATE, "forces before the first deposit");
  if (n < 0) return rp_fail(ctx, RP_EINVAL, "forces: n < 0");
  if (n == 0) return RP_OK;
  if (!x || !y || !ux || !uy || !ex || !ey || !bz || !fx || !fy)
    return rp_fail(ctx, RP_EINVAL, "forces: null array");
  rp_frame Fk = ctx->fh[slot_of(ctx->k, ctx->H)];
  k_forces<<<(unsigned)((n + 255) / 256), 256, 0, ctx->stream>>>(n, x, y, ux, uy, Fk, c.nx, c.ny,
                                                                  1.0 / c.hx, 1.0 / c.hy, bz_ext,
                                                                  ex, ey, bz, fx, fy);
  RP_CHECK_LAUNCH();
  return RP_OK;
}

int rp_kick_impl(rp_ctx* ctx, const double* ux, const double* uy, int64_t n, double qmc,
                 double bz_ext, double frac, double* ox, double* oy) {
  if (n < 0) return rp_fail(ctx, RP_EINVAL, "kick: n < 0");
  if (n == 0) return RP_OK;
  if (!ux || !uy || !ox || !oy) return rp_fail(ctx, RP_EINVAL, "kick: null array");
  const double h = 0.5 * qmc * (frac * ctx->cfg.dt);
  k_kick_external<<<(unsigned)((n + 255) / 256), 256, 0, ctx->stream>>>(n, ux, uy, h, bz_ext, ox, oy);
  RP_CHECK_LAUNCH();
  return RP_OK;
}
