// potentials.cu -- step 2 of the paper's loop: retarded potentials at every grid point
// (Eq. 1-2; Algorithm 1 COMPUTE-POTENTIALS), B200-native.
//
// Kernels (one launch each per call):
//   k_clip       one thread per (point p, subregion j): support clip [A, B] of S_j (R-5),
//                bit-identical to the oracle (IEEE _rn intrinsics, no contraction); emits the
//                scheduling key from the previous step's segment count (the forecast g of
//                P:85-95 used for scheduling only; LPT order).
//   CUB sort     (key, item) -> longest-predicted-first order.
//   k_integrate  persistent warps pull (p, j) items; each warp walks the canonical dyadic
//                GK15 tree of its item depth-first without a stack (R-8..R-12).  Per
//                segment lanes 0..14 build the 15 r' nodes (retarded frame, circle/support
//                arcs, R-5/R-7); then lane l evaluates f (27-point TSC x Lagrange-3 gather,
//                R-6) at theta slot 32r+l for all 15 nodes from a register stencil cache that
//                survives across radially adjacent segments, and the K15/G7 sums are reduced
//                with xor shuffles, so every accept/split decision is warp-uniform.
//   k_reduce     per point, sum the items in j order -> phi, A, err, nseg; counts.
// FP64 throughout.  No tensor cores: the work is an irregular gather stencil,
// not a dense contraction.
#include <math_constants.h>
#include <cub/device/device_radix_sort.cuh>
#include <math.h>

#include "rp_internal.cuh"

int rp_ensure_cub_tmp(rp_ctx* ctx, size_t bytes);

namespace {

// QUADPACK qk15 nodes / Kronrod weights / Gauss-7 weights (R-8)
__constant__ double c_xgk[8] = {
    0.991455371120812639206854697526329, 0.949107912342758524526189684047851,
    0.864864423359769072789712788640926, 0.741531185599394439863864773280788,
    0.586087235467691130294144845693013, 0.405845151377397166906606412076961,
    0.207784955007898467600689403773245, 0.000000000000000000000000000000000};
__constant__ double c_wgk[8] = {
    0.022935322010529224963732008058970, 0.063092092629978553290700663189204,
    0.104790010322250183839876322541518, 0.140653259715525918745189590510238,
    0.169004726639267902826583426598550, 0.190350578064785409913256402421014,
    0.204432940075298892414161999234649, 0.209482141084727828012999174891714};
__constant__ double c_wg[4] = {
    0.129484966168869693270611432679082, 0.279705391489276667901467771423780,
    0.381830050505118944950369775488975, 0.417959183673469387755102040816327};

enum : int { C_ITEMS = 0, C_NEXT = 1, C_EVALS = 2, C_SEGS = 3, C_LEAVES = 4, C_CAPPED = 5,
             C_TIES = 6, C_MAXLEV = 7, C_NODES = 8, C_NOUT = 9, C_SKIP = 10, C_UNITS = 11,
             C_NEXT_U = 12, C_COUNT = 16 };
constexpr int kUnitShift = 20;  // unit key = item << 20 | index of the subtree root at its level
constexpr int kGridVar = 4;  // grid evaluation loop: software-pipelined rounds (6 = Lagrange-3;
                             // 5 / 7: the same recording the accepted leaves, R-26b)
constexpr int kUnitBudget = 64;  // subtree units per near-field item (DFS order)
constexpr uint32_t kEmptyKey = 0xFFFFFFFFu;  // schedule key of an item without support

constexpr double kTwoPi = 6.283185307179586476925286766559;
constexpr int kMaxArcs = 8;
constexpr int kWarps = 1;  // warps per CTA of k_integrate (1: the warp's shared block sits at
                            // a constant address, no per-iteration warp-index arithmetic)

struct Params {
  int nx, ny, PX, npts, kmax, kap, k, H, n_theta, max_depth, n_root, rule, variant, interp;
  double hx, hy, inv_hx, inv_hy, cdt, tau, R;
  double inv_n_theta;        // 1/N when N is a power of two (x/N = x * (1/N) exactly), else 0
  double grid_extent;        // max(nx hx, ny hy): the near-field root scale (R-12b)
  size_t slot_doubles;
  const double* ring;        // padded ring, slot 0 node (-PAD, -PAD)
  const rp_frame* frames;    // [H]
  const double* amp;         // [H] analytic amplitudes
  // Predictive-RP (R-26): merged partition lists per (cluster, j) and the point clusters;
  // bp_off == nullptr selects the canonical roots
  const double* bp;
  const int64_t* bp_off;
  const int32_t* cluster;
  // adaptive partitioning (R-26b): every accepted leaf appended as (a, b, item, 0)
  double4* leaf_rec;
  unsigned long long* leaf_count;
  long long leaf_cap;
  // subtree work units (deep trees split at a fixed level, see k_integrate)
  int split_level;                  // 0: off
  int split_j;                      // only subregions j < split_j are split (the near field)
  int unit_budget;                  // at most this many units per item (the first in DFS order)
  int32_t* unit_ndef;               // [npts * split_j] units deferred by each near-field item
  unsigned long long* unit_key;     // [slots] item << kUnitShift | ix, item-major fixed slots
  const int32_t* unit_order;        // unit launch: the units, longest-predicted-first
  double4* unit_val;
  int4* unit_cnt;
  uint2* unit_aux;
  // analytic source
  double sx0, sy0, swidth, sq, sbx, sby;
};

struct Item {
  double px, py;              // mesh point, lab
  int j;
  rp_frame F0, F1, F2;        // frames of levels k-j-2, k-j-1, k-j
  const double* g0;           // level grids at padded node (0, 0)
  const double* g1;
  const double* g2;
  double a0, a1, a2;          // analytic amplitudes
  double U0, U1, V0, V1;      // rectangle support (grid / gauss), frame-local
};

// ------------------------------------------------------------- bit-exact geometry
// These mirror the arithmetic order of the definition with IEEE
// round-to-nearest intrinsics so clip limits and segment endpoints are reproducible.
__device__ __forceinline__ void lag3(double t, double& w0, double& w1, double& w2) {
  w0 = __dmul_rn(__dmul_rn(0.5, t), __dsub_rn(t, 1.0));
  w1 = __dsub_rn(1.0, __dmul_rn(t, t));
  w2 = __dmul_rn(__dmul_rn(0.5, t), __dadd_rn(t, 1.0));
}

__device__ __forceinline__ double lerp3(double x0, double x1, double x2, double w0, double w2) {
  return __dadd_rn(__dadd_rn(x1, __dmul_rn(w0, __dsub_rn(x0, x1))), __dmul_rn(w2, __dsub_rn(x2, x1)));
}

// frame-local centre of the circle about p at the retarded time of radius r (R-7)
__device__ __forceinline__ void centre_at(const Item& it, const Params& P, double r, double& cu,
                                          double& cv, double& w0, double& w1, double& w2) {
  double t = __dsub_rn((double)(it.j + 1), __ddiv_rn(r, P.cdt));
  lag3(t, w0, w1, w2);
  double ox = lerp3(it.F0.ox, it.F1.ox, it.F2.ox, w0, w2);
  double oy = lerp3(it.F0.oy, it.F1.oy, it.F2.oy, w0, w2);
  double c = lerp3(it.F0.cos_psi, it.F1.cos_psi, it.F2.cos_psi, w0, w2);
  double s = lerp3(it.F0.sin_psi, it.F1.sin_psi, it.F2.sin_psi, w0, w2);
  double dx = __dsub_rn(it.px, ox), dy = __dsub_rn(it.py, oy);
  cu = __dadd_rn(__dmul_rn(c, dx), __dmul_rn(s, dy));
  cv = __dadd_rn(__dmul_rn(-s, dx), __dmul_rn(c, dy));
}

template <int KIND>
__device__ __forceinline__ void support_d2(const Item& it, const Params& P, double cu, double cv,
                                           double& dmin2, double& dmax2) {
  if (KIND == RP_SRC_DISK) {
    double ex = __dsub_rn(cu, P.sx0), ey = __dsub_rn(cv, P.sy0);
    double s = __dsqrt_rn(__dadd_rn(__dmul_rn(ex, ex), __dmul_rn(ey, ey)));
    double lo = __dsub_rn(s, P.swidth);
    lo = lo > 0.0 ? lo : 0.0;
    double hi = __dadd_rn(s, P.swidth);
    dmin2 = __dmul_rn(lo, lo);
    dmax2 = __dmul_rn(hi, hi);
    return;
  }
  double ex = 0.0, ey = 0.0;
  if (cu < it.U0) ex = __dsub_rn(it.U0, cu); else if (cu > it.U1) ex = __dsub_rn(cu, it.U1);
  if (cv < it.V0) ey = __dsub_rn(it.V0, cv); else if (cv > it.V1) ey = __dsub_rn(cv, it.V1);
  dmin2 = __dadd_rn(__dmul_rn(ex, ex), __dmul_rn(ey, ey));
  double a = fabs(__dsub_rn(cu, it.U0)), b = fabs(__dsub_rn(cu, it.U1));
  double fx = a > b ? a : b;
  a = fabs(__dsub_rn(cv, it.V0));
  b = fabs(__dsub_rn(cv, it.V1));
  double fy = a > b ? a : b;
  dmax2 = __dadd_rn(__dmul_rn(fx, fx), __dmul_rn(fy, fy));
}

template <int KIND>
__device__ __forceinline__ void dists_at(const Item& it, const Params& P, double r, double& dmin2,
                                         double& dmax2) {
  double cu, cv, w0, w1, w2;
  centre_at(it, P, r, cu, cv, w0, w1, w2);
  support_d2<KIND>(it, P, cu, cv, dmin2, dmax2);
}

template <int KIND>
__device__ void setup_item(Item& it, const Params& P, int p, int j) {
  int ix = p % P.nx, iy = p / P.nx;
  const rp_frame Fk = P.frames[slot_of_dev(P.k, P.H)];
  double u = __dmul_rn((double)ix, P.hx), v = __dmul_rn((double)iy, P.hy);
  it.px = __dsub_rn(__dadd_rn(Fk.ox, __dmul_rn(u, Fk.cos_psi)), __dmul_rn(v, Fk.sin_psi));
  it.py = __dadd_rn(__dadd_rn(Fk.oy, __dmul_rn(u, Fk.sin_psi)), __dmul_rn(v, Fk.cos_psi));
  it.j = j;
  int s0 = slot_of_dev(P.k - j - 2, P.H), s1 = slot_of_dev(P.k - j - 1, P.H),
      s2 = slot_of_dev(P.k - j, P.H);
  it.F0 = P.frames[s0];
  it.F1 = P.frames[s1];
  it.F2 = P.frames[s2];
  size_t off = (size_t)4 * (RP_PAD * P.PX + RP_PAD);
  it.g0 = P.ring + (size_t)s0 * P.slot_doubles + off;
  it.g1 = P.ring + (size_t)s1 * P.slot_doubles + off;
  it.g2 = P.ring + (size_t)s2 * P.slot_doubles + off;
  if (KIND != RP_SRC_GRID) {
    it.a0 = P.amp[s0];
    it.a1 = P.amp[s1];
    it.a2 = P.amp[s2];
  } else {
    it.a0 = it.a1 = it.a2 = 1.0;
  }
  if (KIND == RP_SRC_GAUSS) {
    double w8 = __dmul_rn(8.0, P.swidth);
    it.U0 = __dsub_rn(P.sx0, w8); it.U1 = __dadd_rn(P.sx0, w8);
    it.V0 = __dsub_rn(P.sy0, w8); it.V1 = __dadd_rn(P.sy0, w8);
  } else {
    it.U0 = __dmul_rn(-1.5, P.hx);
    it.U1 = __dmul_rn(__dadd_rn((double)P.nx, 0.5), P.hx);
    it.V0 = __dmul_rn(-1.5, P.hy);
    it.V1 = __dmul_rn(__dadd_rn((double)P.ny, 0.5), P.hy);
  }
}

// ------------------------------------------------------------- k_clip
// Forecast of the segments of item (p, j) from last step's counts (scheduling only).
__device__ __forceinline__ unsigned forecast(const uint16_t* __restrict__ cost, int p, int j,
                                             int nx, int ny, int kmax, int policy, int knn) {
  if (policy != RP_SCHED_KNN || knn <= 1) return cost[(size_t)p * kmax + j];
  // kNN regression over the comoving mesh: k nearest nodes in index space
  const int ix = p % nx, iy = p / nx;
  const int rad = knn >= 25 ? 2 : 1;
  unsigned sum = 0, cnt = 0;
  for (int dy = -rad; dy <= rad; ++dy)
    for (int dx = -rad; dx <= rad; ++dx) {
      if (knn == 5 && dx != 0 && dy != 0) continue;  // 4-neighbour cross + centre
      const int x = ix + dx, y = iy + dy;
      if (x < 0 || x >= nx || y < 0 || y >= ny) continue;
      sum += cost[((size_t)y * nx + x) * kmax + j];
      ++cnt;
    }
  return cnt ? (sum + cnt / 2) / cnt : 0u;
}

template <int KIND>
__global__ void k_clip(Params P, const int32_t* __restrict__ owner, int rank,
                       const uint16_t* __restrict__ cost_prev, int policy, int knn,
                       double2* __restrict__ AB,
                       uint32_t* __restrict__ key, int32_t* __restrict__ iota,
                       unsigned long long* __restrict__ counters) {
  int64_t id = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  int64_t total = (int64_t)P.npts * P.kmax;
  if (id >= total) return;
  iota[id] = (int32_t)id;
  int p = (int)(id / P.kmax), j = (int)(id % P.kmax);
  uint32_t kk = kEmptyKey;
  double A = 0.0, B = 0.0;
  if (j < P.kap && (owner == nullptr || owner[p] == rank)) {
    Item it;
    setup_item<KIND>(it, P, p, j);
    double a = __dmul_rn((double)j, P.cdt), b = __dmul_rn((double)(j + 1), P.cdt);
    double dmn, dmx;
    bool empty = false;
    dists_at<KIND>(it, P, b, dmn, dmx);
    if (dmn > __dmul_rn(b, b)) empty = true;
    if (!empty) {
      dists_at<KIND>(it, P, a, dmn, dmx);
      if (dmx < __dmul_rn(a, a)) empty = true;
    }
    if (!empty) {
      if (dmn <= __dmul_rn(a, a)) {
        A = a;
      } else {
        double lo = a, hi = b;
        for (int t = 0; t < 64; ++t) {
          double m = __dmul_rn(0.5, __dadd_rn(lo, hi));
          dists_at<KIND>(it, P, m, dmn, dmx);
          if (dmn <= __dmul_rn(m, m)) hi = m; else lo = m;
        }
        A = hi;
      }
      dists_at<KIND>(it, P, b, dmn, dmx);
      if (dmx >= __dmul_rn(b, b)) {
        B = b;
      } else {
        double lo = a, hi = b;
        for (int t = 0; t < 64; ++t) {
          double m = __dmul_rn(0.5, __dadd_rn(lo, hi));
          dists_at<KIND>(it, P, m, dmn, dmx);
          if (dmx >= __dmul_rn(m, m)) lo = m; else hi = m;
        }
        B = lo;
      }
      if (A < B) {
        // no forecast yet (first step): the near-field subregion S_0 carries most of the work
        // (DESIGN.md sec. 3), so run it first; later steps use last step's counts
        unsigned c = cost_prev ? forecast(cost_prev, p, j, P.nx, P.ny, P.kmax, policy, knn)
                               : (policy == RP_SCHED_INDEX ? 0u : (j == 0 ? 1u : 0u));
        kk = 0xFFFEu - (c < 0xFFFEu ? c : 0xFFFEu);
        // subregion-major order (j ascending, longest-predicted-first within j): concurrent
        // warps share the 3 history levels of one subregion, so the slab stays L2-resident
        // when the ring does not fit in L2 (configs 4-5)
        if (policy == RP_SCHED_SUBREGION) kk |= (uint32_t)min(j, 0xFFFE) << 16;
      }
    }
  }
  AB[id] = make_double2(A, B);
  key[id] = kk;
  // count items: warp aggregate then one atomic per warp (integer -> deterministic)
  unsigned m = __ballot_sync(__activemask(), kk != kEmptyKey);
  if ((threadIdx.x & 31) == (__ffs(__activemask()) - 1) && m)
    atomicAdd(&counters[C_ITEMS], (unsigned long long)__popc(m));
}

// ------------------------------------------------------------- integrand (analytic sources)
template <int KIND>
__device__ __forceinline__ void integrand(const Item& it, const Params& P, double u, double v,
                                          double w0, double w1, double w2, double& f0,
                                          double& f1, double& f2) {
  double amp = w0 * it.a0 + w1 * it.a1 + w2 * it.a2;
  double rho;
  if (KIND == RP_SRC_GAUSS) {
    double ex = u - P.sx0, ey = v - P.sy0, sg = P.swidth;
    rho = P.sq / (kTwoPi * sg * sg) * exp(-(ex * ex + ey * ey) / (2.0 * sg * sg));
  } else {
    rho = P.sq;
  }
  rho *= amp;
  f0 = rho;
  f1 = rho * P.sbx;
  f2 = rho * P.sby;
}

// ------------------------------------------------------------- bounded sincos
// sin/cos for |x| <= 8 pi: Cody-Waite reduction by pi/2 with a two-term constant (k <= 16 is
// exact enough for ulp-level accuracy) and the classic fdlibm minimax kernels on
// [-pi/4, pi/4].  No Payne-Hanek slow path, so it inlines small.
// fdlibm __kernel_sin / __kernel_cos coefficients, in the constant bank so every DFMA takes
// them as a c[] operand (no per-call uniform-register moves)
__constant__ double c_sinp[6] = {1.58969099521155010221e-10, -2.50507602534068634195e-08,
                                 2.75573137070700676789e-06, -1.98412698298579493134e-04,
                                 8.33333333332248946124e-03, -1.66666666666666324348e-01};
__constant__ double c_cosp[6] = {-1.13596475577881948265e-11, 2.08757232129817482790e-09,
                                 -2.75573143513906633035e-07, 2.48015872894767294178e-05,
                                 -1.38888888888741095749e-03, 4.16666666666666019037e-02};
__constant__ double c_pio2[3] = {0.63661977236758134308, 1.5707963267948965580,
                                 6.1232339957367658e-17};  // 2/pi, pi/2 = hi + lo

// Round-to-integer through the FP64 adder: for |y| < 2^51, y + 1.5 * 2^52 rounds y to an
// integer in the unit of the last place (IEEE mode of the add), the low word of the sum is that
// integer (two's complement) and the sum minus the constant is it as a double -- exact, and on
// the FP64 pipe instead of the variable-latency FRND / F2I conversions.
constexpr double kRoundMagic = 6755399441055744.0;  // 1.5 * 2^52

__device__ __forceinline__ void sincos_b(double x, double* s, double* c) {
  const double kk = __dadd_rn(__dmul_rn(x, c_pio2[0]), kRoundMagic);  // rint(x * 2/pi) + magic
  const double k = __dsub_rn(kk, kRoundMagic);
  double r = fma(-k, c_pio2[1], x);
  r = fma(-k, c_pio2[2], r);
  const double z = r * r;
  double ps = fma(z, c_sinp[0], c_sinp[1]);
  ps = fma(z, ps, c_sinp[2]);
  ps = fma(z, ps, c_sinp[3]);
  ps = fma(z, ps, c_sinp[4]);
  ps = fma(z, ps, c_sinp[5]);
  const double sr = fma(r * z, ps, r);
  double pc = fma(z, c_cosp[0], c_cosp[1]);
  pc = fma(z, pc, c_cosp[2]);
  pc = fma(z, pc, c_cosp[3]);
  pc = fma(z, pc, c_cosp[4]);
  pc = fma(z, pc, c_cosp[5]);
  const double cr = fma(z * z, pc, fma(-0.5, z, 1.0));
  const int q = __double2loint(kk) & 3;
  const double ss = (q & 1) ? cr : sr, cc = (q & 1) ? sr : cr;
  *s = (q & 2) ? -ss : ss;
  *c = ((q + 1) & 2) ? -cc : cc;
}

// ------------------------------------------------------------- arcs (R-5)
__device__ __forceinline__ bool in_rect(double u, double v, const Item& it) {
  return u >= it.U0 && u <= it.U1 && v >= it.V0 && v <= it.V1;
}

// arcs of circle (cu, cv; r) inside the support; returns -1 (full circle) or the count,
// writing (theta1, dtheta = (theta2 - theta1) / N) pairs.
template <int KIND>
__device__ int arcs(const Item& it, const Params& P, double cu, double cv, double r,
                    double* th1, double* dth) {
  const double N = (double)P.n_theta;
  if (KIND == RP_SRC_DISK) {
    double ex = P.sx0 - cu, ey = P.sy0 - cv;
    double s = sqrt(ex * ex + ey * ey), a = P.swidth;
    if (s + r <= a) return -1;
    if (r >= s + a || s >= r + a) return 0;
    double ph = atan2(ey, ex);
    double al = acos((r * r + s * s - a * a) / (2.0 * r * s));
    th1[0] = ph - al;
    dth[0] = ((ph + al) - (ph - al)) / N;
    return 1;
  }
  // Crossings of the circle with the 4 edge lines that lie on the edge.  Edge e's two
  // crossings sit in fixed slots 2e, 2e + 1 (+inf when absent), sorted by a 19-comparator
  // network and consumed through a register shift, so nothing goes to local memory.
  double t[8];
  int n = 0;
  const double rinv = 1.0 / r;
#pragma unroll
  for (int e = 0; e < 4; ++e) {  // the 4 edges are independent: unrolled for ILP
    t[2 * e] = t[2 * e + 1] = CUDART_INF;
    const bool vert = e < 2;
    const double edge = e == 0 ? it.U0 : e == 1 ? it.U1 : e == 2 ? it.V0 : it.V1;
    const double de = __dsub_rn(edge, vert ? cu : cv);
    double d = de * rinv;
    // near a tangency (|d| -> 1) whether the circle crosses the edge -- full circle
    // (trapezoid) or arc (Simpson), R-11 -- is decided by the last bit of d: there it is the
    // one IEEE division (edge - c) / r of the oracle, so both sides decide alike (R-19)
    if (fabs(d) > 0.9999) d = __ddiv_rn(de, r);
    if (!(fabs(d) < 1.0)) continue;
    const double h = r * sqrt(1.0 - d * d);  // r sin(acos d) = r cos(asin d)
    const double lo = vert ? it.V0 : it.U0, hi = vert ? it.V1 : it.U1;
    const double o1 = (vert ? cv : cu) + h, o2 = (vert ? cv : cu) - h;
    double c1, c2;
    if (vert) {
      c1 = acos(d);
      c2 = kTwoPi - c1;
    } else {
      const double be = asin(d);
      c1 = be < 0.0 ? be + kTwoPi : be;
      c2 = M_PI - be;
    }
    if (o1 >= lo && o1 <= hi) { t[2 * e] = c1; ++n; }
    if (o2 >= lo && o2 <= hi) { t[2 * e + 1] = c2; ++n; }
  }
  if (n == 0) return in_rect(cu + r, cv, it) ? -1 : 0;
  constexpr int kNet[19][2] = {{0, 1}, {2, 3}, {4, 5}, {6, 7}, {0, 2}, {1, 3}, {4, 6},
                               {5, 7}, {1, 2}, {5, 6}, {0, 4}, {1, 5}, {2, 6}, {3, 7},
                               {2, 4}, {3, 5}, {1, 2}, {3, 4}, {5, 6}};
#pragma unroll
  for (int c = 0; c < 19; ++c) {
    const double x = t[kNet[c][0]], y = t[kNet[c][1]];
    const bool sw = y < x;
    t[kNet[c][0]] = sw ? y : x;
    t[kNet[c][1]] = sw ? x : y;
  }
  // unique crossings u_0 < u_1 < ...; keep the intervals (u_i, u_{i+1}) and
  // (u_last, u_0 + 2 pi) whose midpoint lies inside the rectangle
  int na = 0;
  const double first = t[0];
  double prev = first;
#pragma unroll 1
  for (int i = 1; i <= n; ++i) {
    const double cur = i < n ? t[1] : first + kTwoPi;
#pragma unroll
    for (int q = 1; q < 7; ++q) t[q] = t[q + 1];
    if (i < n && cur == prev) continue;
    double sm, cm;
    sincos_b(0.5 * (prev + cur), &sm, &cm);
    if (in_rect(cu + r * cm, cv + r * sm, it)) {
      th1[na] = prev;
      dth[na] = P.inv_n_theta != 0.0 ? (cur - prev) * P.inv_n_theta : (cur - prev) / N;
      ++na;
    }
    prev = cur;
  }
  return na;
}

// ------------------------------------------------------------- k_integrate
struct __align__(16) NodeRec {
  double r, cu, cv, w0, w1, w2, wk, wg;  // r', frame-local centre, time weights, hw*w_GK, hw*w_G7
};

constexpr int kNoCell = -0x7fffffff;  // geometry record of a slot a node does not have

struct WarpSmem {
  Item it;  // per-item geometry, kept in shared memory to free registers for the eval loop
  NodeRec node[16];
  double th1[16][kMaxArcs], dth[16][kMaxArcs];
  int na[16], cnt[16];
};

// 256-bit read-only load of one padded node record (rho, rho*bx, rho*by, 0): sm_100
// LDG.E.ENL2.256, one instruction per stencil node.
__device__ __forceinline__ void ldg_node(const double* p, double& a, double& b, double& c) {
  double d;
  asm("ld.global.nc.v4.f64 {%0,%1,%2,%3}, [%4];" : "=d"(a), "=d"(b), "=d"(c), "=d"(d) : "l"(p));
}

// Analytic sources (test path): theta slot e of the r' nodes n0 .. n1-1 of the
// current segment, evaluated in closed form (no stencil).
template <int KIND>
__device__ __forceinline__ void eval_nodes(const Item& it, const Params& P, const WarpSmem& S,
                                           const double2* __restrict__ trig_full, int e, int n0,
                                           int n1, int N, double wfull, double third,
                                           double& k0, double& k1, double& k2, double& g0,
                                           double& g1, double& g2) {
  // the full-circle node of slot e is the same for every r' node: one load per call
  const double2 trf = __ldg(trig_full + (e < N ? e : 0));
#pragma unroll 3
  for (int n = n0; n < n1; ++n) {
    if (e >= S.cnt[n]) continue;
    const int na = S.na[n];
    const NodeRec& nd = S.node[n];
    double cs, sn, w;
    if (na < 0) {
      cs = trf.x;
      sn = trf.y;
      w = wfull;
    } else {
      int q = 0, mm = e;
      while (mm > N) {  // arc index without a division (one arc in the common case)
        mm -= N + 1;
        ++q;
      }
      const double d = S.dth[n][q];
      sincos_b(S.th1[n][q] + (double)mm * d, &sn, &cs);
      const double coef = (mm == 0 || mm == N) ? 1.0 : ((mm & 1) ? 4.0 : 2.0);
      w = coef * d * third;
    }
    const double u = nd.cu + nd.r * cs, v = nd.cv + nd.r * sn;
    double f0, f1, f2;
    integrand<KIND>(it, P, u, v, nd.w0, nd.w1, nd.w2, f0, f1, f2);
    const double wk = w * nd.wk;
    k0 += wk * f0; k1 += wk * f1; k2 += wk * f2;
    if ((n & 1) || P.rule == RP_RULE_SIMPSON) {  // G7: Gauss nodes only (warp-uniform n)
      const double wg = w * nd.wg;
      g0 += wg * f0; g1 += wg * f1; g2 += wg * f2;
    }
  }
}

// ---- software-pipelined round (VAR 4): geometry of node n+1 and the contraction of node n
// form one basic block, so the long sincos / floor chains of the next point fill the latency
// gaps of the current contraction (2 warps per scheduler cannot hide them otherwise).
struct Geo {
  double dx, dy, w;
  int cell;
};

// Branch-free geometry of theta slot e of r' node n (FULL: full circle, uniform per node).
template <bool FULL, bool LAG>
__device__ __forceinline__ Geo geom_point(const Params& P, const WarpSmem& S, double2 trf, int e,
                                          int n, int N, double wfull, double third,
                                          float inv_n1) {
  const bool valid = e < S.cnt[n];
  double cs, sn, w;
  if (FULL) {
    cs = trf.x;
    sn = trf.y;
    w = wfull;
  } else {
    // slot e -> arc q, interior Simpson node mm = 1 .. N-1: the end nodes mm = 0, N of an arc
    // lie on the support boundary, where the zero-padded TSC stencil vanishes (R-24) and the
    // Lagrange-3 integrand takes its limit from outside, 0 (R-25b)
    const int ec = valid ? e : 0;
    // arc index trunc((ec + 1/2) / (N - 1)), exact for e < 2^20 (the quotient stays >= 1/(2N)
    // from an integer); truncated by an FP32 add in round-toward-zero (no F2I)
    const float qf = __fadd_rz(fmaf((float)ec, inv_n1, 0.5f * inv_n1), 12582912.0f);
    const int q = __float_as_int(qf) - 0x4B400000;
    const int mm = ec - q * (N - 1) + 1;
    const double d = S.dth[n][q];
    const double mmd = __dsub_rn(__hiloint2double(0x43300000, mm), 4503599627370496.0);  // (double)mm
    sincos_b(S.th1[n][q] + mmd * d, &sn, &cs);
    const double coef = (mm & 1) ? 4.0 : 2.0;
    w = coef * d * third;
  }
  const NodeRec& nd = S.node[n];
  const double u = nd.cu + nd.r * cs, v = nd.cv + nd.r * sn;
  // nearest node (ix, iy) = floor(t + 1/2) and the offset t - floor(t + 1/2), t = u / h: the
  // floor as a round-down add of the magic constant (see sincos_b; no FRND / F2I)
  const double sx = __dadd_rd(fma(u, P.inv_hx, 0.5), kRoundMagic);
  const double sy = __dadd_rd(fma(v, P.inv_hy, 0.5), kRoundMagic);
  const double fx = __dsub_rn(sx, kRoundMagic), fy = __dsub_rn(sy, kRoundMagic);
  const int ix = min(max(__double2loint(sx), -2), P.nx + 1);
  const int iy = min(max(__double2loint(sy), -2), P.ny + 1);
  // a slot the node does not have evaluates slot 0's (finite) point with weight 0 and no refill
  Geo g;
  g.dx = fma(u, P.inv_hx, -fx);
  g.dy = fma(v, P.inv_hy, -fy);
  g.w = valid ? (LAG ? w : 0.25 * w) : 0.0;  // 0.25 undoes the 2 x 2 scaling of the TSC weights
  g.cell = valid ? (iy - 1) * P.PX + (ix - 1) : kNoCell;
  return g;
}

__device__ __forceinline__ void refill(const Item& it, size_t rs, int cell,
                                       double (&st)[3][9][3]) {
  const size_t base = (size_t)4 * (ptrdiff_t)cell;
  const double* g[3] = {it.g0 + base, it.g1 + base, it.g2 + base};
#pragma unroll
  for (int l = 0; l < 3; ++l)
#pragma unroll
    for (int b = 0; b < 3; ++b) {
      const double* row = g[l] + b * rs;
#pragma unroll
      for (int a = 0; a < 3; ++a)
        ldg_node(row + 4 * a, st[l][3 * b + a][0], st[l][3 * b + a][1], st[l][3 * b + a][2]);
    }
}

// 27-node x 3-component contraction at one point -> (f0, f1, f2)
template <bool LAG>
__device__ __forceinline__ void contract_point(const Geo& g, const NodeRec& nd,
                                               const double (&st)[3][9][3], double& f0,
                                               double& f1, double& f2) {
  const double dx = g.dx, dy = g.dy;
  double wx[3], wy[3];
  if (LAG) {  // quadratic Lagrange at nodes -1, 0, +1 (R-25)
    const double hx = 0.5 * dx, hy = 0.5 * dy;
    wx[0] = hx * (dx - 1.0); wx[1] = fma(-dx, dx, 1.0); wx[2] = hx * (dx + 1.0);
    wy[0] = hy * (dy - 1.0); wy[1] = fma(-dy, dy, 1.0); wy[2] = hy * (dy + 1.0);
  } else {  // 2 x TSC
    const double ax = 0.5 - dx, bx = 0.5 + dx, ay = 0.5 - dy, by = 0.5 + dy;
    wx[0] = ax * ax; wx[1] = fma(-2.0 * dx, dx, 1.5); wx[2] = bx * bx;
    wy[0] = ay * ay; wy[1] = fma(-2.0 * dy, dy, 1.5); wy[2] = by * by;
  }
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
  f0 = nd.w0 * s[0][0] + nd.w1 * s[1][0] + nd.w2 * s[2][0];
  f1 = nd.w0 * s[0][1] + nd.w1 * s[1][1] + nd.w2 * s[2][1];
  f2 = nd.w0 * s[0][2] + nd.w1 * s[1][2] + nd.w2 * s[2][2];
}

template <bool LAG>
__device__ __forceinline__ void pipelined_round(const Item& it, const Params& P,
                                                const WarpSmem& S,
                                                const double2* __restrict__ trig_full, int e,
                                                int nn, int N, double wfull, double third,
                                                double (&st)[3][9][3], int& ccell, double& k0,
                                                double& k1, double& k2, double& g0, double& g1,
                                                double& g2, unsigned fullmask,
                                                unsigned gmask) {
  const size_t rs = (size_t)4 * P.PX;
  const float inv_n1 = 1.0f / (float)(N - 1);  // arc slots per arc (R-24, R-25b)
  const double2 trf = __ldg(trig_full + (e < N ? e : 0));
  Geo cur = (fullmask & 1) ? geom_point<true, LAG>(P, S, trf, e, 0, N, wfull, third, inv_n1)
                        : geom_point<false, LAG>(P, S, trf, e, 0, N, wfull, third, inv_n1);
#pragma unroll 1
  for (int n = 0; n < nn; ++n) {
    if (cur.cell != kNoCell && cur.cell != ccell) {
      ccell = cur.cell;
      refill(it, rs, cur.cell, st);
    }
    const NodeRec& nd = S.node[n];
    double f0, f1, f2;
    Geo nxt;
    if (n + 1 < nn && ((fullmask >> (n + 1)) & 1)) {
      nxt = geom_point<true, LAG>(P, S, trf, e, n + 1, N, wfull, third, inv_n1);
      contract_point<LAG>(cur, nd, st, f0, f1, f2);
    } else if (n + 1 < nn) {
      nxt = geom_point<false, LAG>(P, S, trf, e, n + 1, N, wfull, third, inv_n1);
      contract_point<LAG>(cur, nd, st, f0, f1, f2);
    } else {
      nxt = cur;
      contract_point<LAG>(cur, nd, st, f0, f1, f2);
    }
    const double wk = cur.w * nd.wk;
    k0 += wk * f0; k1 += wk * f1; k2 += wk * f2;
    if ((gmask >> n) & 1) {  // G7: Gauss nodes only (warp-uniform n)
      const double wg = cur.w * nd.wg;
      g0 += wg * f0; g1 += wg * f1; g2 += wg * f2;
    }
    cur = nxt;
  }
}

__device__ __forceinline__ double warp_sum(double v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  return v;
}

// VAR 0: analytic sources (eval_nodes); VAR 4: grid, TSC, software-pipelined rounds with the
// register stencil cache; VAR 6: the same with the Lagrange-3 spatial weights (R-25).
// UNIT = false: the (point, subregion) items in forecast order.  With P.split_level = L > 0
// a segment at level L - 1 of a near-field item (j < split_j) that splits does not descend:
// its two children become subtree work units -- written to the item's own fixed slots
// (item-major, at most unit_budget per item, in DFS order) -- and the walk goes on as if the
// segment were finished.  The
// tree is the canonical one -- only nodes it reaches are deferred -- but the deep near-field
// trees (thousands of segments, fanning out below level ~8) no longer bound the kernel (and an
// N-GPU shard) by one warp's walk.  UNIT = true: the units, each walked from its root at
// level L until the walk climbs back to L; per-unit results are merged into their items in
// (item, subtree) order (k_merge_units), so results are deterministic for any N.
template <int KIND, int VAR, bool UNIT = false>
__global__ void __launch_bounds__(32 * kWarps) k_integrate(
    Params P, const int32_t* __restrict__ order, const double2* __restrict__ AB,
    const double2* __restrict__ trig_full, double4* __restrict__ item_val,
    int4* __restrict__ item_cnt, uint2* __restrict__ item_aux,
    unsigned long long* __restrict__ counters) {
  // one warp per CTA: its per-item block is a static shared variable (a fixed shared address,
  // no per-access window arithmetic)
  __shared__ WarpSmem smem[kWarps];
  const int lane = threadIdx.x & 31;
  WarpSmem& S = smem[kWarps == 1 ? 0 : (threadIdx.x >> 5)];
  const unsigned long long n_items = counters[UNIT ? C_UNITS : C_ITEMS];
  const int N = P.n_theta;
  const double Nd = (double)N;
  const double wfull = kTwoPi / Nd;
  const double third = 1.0 / 3.0;
  for (;;) {
    unsigned long long idx = 0;
    if (lane == 0) idx = atomicAdd(&counters[UNIT ? C_NEXT_U : C_NEXT], 1ULL);
    idx = __shfl_sync(0xffffffffu, idx, 0);
    if (idx >= n_items) break;
    const int uidx = UNIT ? P.unit_order[idx] : 0;
    const unsigned long long ukey = UNIT ? P.unit_key[uidx] : 0ULL;
    const int item = UNIT ? (int)(ukey >> kUnitShift) : order[idx];
    const int p = item / P.kmax, j = item % P.kmax;
    const double2 ab = AB[item];
    // roots of the item's trees: the n_root halves of its support [A, B] (canonical), or the
    // intervals of its cluster's merged partition of S_j cut to [A, B] (Predictive-RP,
    // Algorithm 1 lines 13-24, R-26); all lanes walk the list in step (uniform loads)
    long long rt = 0, rt_end = 0;  // next interval [bp[rt], bp[rt + 1]], rt < rt_end
    if (KIND == RP_SRC_GRID && P.bp_off && !UNIT) {
      const long long li = (long long)P.cluster[p] * P.kmax + j;
      rt = P.bp_off[li];
      rt_end = P.bp_off[li + 1] - 1;
      if (rt_end - rt < 1) {
        rt = rt_end = 0;
      } else {  // first interval that ends beyond A
        long long lo = rt, hi = rt_end - 1;
        while (lo < hi) {
          const long long mid = (lo + hi) >> 1;
          if (P.bp[mid + 1] > ab.x) hi = mid; else lo = mid + 1;
        }
        rt = lo;
      }
    }
    const bool pred = rt < rt_end;
    double A = ab.x, BA = __dsub_rn(ab.y, ab.x);
    // R-10's tolerance (tau ((B - A) 2^-l)) / R = ((tau (B - A)) / R) 2^-l exactly (power-of-two
    // scalings commute with rounding; tol stays far above the subnormals): one division per root
    double tol0 = __ddiv_rn(__dmul_rn(P.tau, BA), P.R);
    if (pred) {  // first non-empty cut interval (one exists: the list covers S_j, [A, B] in S_j)
      for (; rt < rt_end; ++rt) {
        const double a = fmax(P.bp[rt], ab.x), b = fmin(P.bp[rt + 1], ab.y);
        if (a < b) {
          A = a; BA = __dsub_rn(b, a); ++rt;
          tol0 = __ddiv_rn(__dmul_rn(P.tau, BA), P.R);
          break;
        }
      }
    }
    __syncwarp();
    if (lane == 0) setup_item<KIND>(S.it, P, p, j);
    __syncwarp();
    const Item& it = S.it;

    double s_phi = 0.0, s_ax = 0.0, s_ay = 0.0, s_err = 0.0;
    double st[3][9][3];                      // per-lane stencil cache (valid for this item's levels)
    int ccell = kNoCell;  // cached cell of the two-pass rounds (empty cache reads as zeros)
    if (KIND == RP_SRC_GRID && VAR >= 4) {
#pragma unroll
      for (int l = 0; l < 3; ++l)
#pragma unroll
        for (int i = 0; i < 9; ++i) st[l][i][0] = st[l][i][1] = st[l][i][2] = 0.0;
    }
    int nseg = 0, nleaf = 0, capped = 0, ties = 0, maxlev = 0, ndef = 0;
    unsigned evals = 0, nskip = 0;
    // canonical roots (R-12b): the n_root = 1, 2 or 4 equal pieces of [A, B] (levels 0, 1, 2);
    // with n_root = 2 the near field S_0 starts from its quarters
    // the near field S_0 (n_root 2 or 4): the 2^L pieces no longer than an eighth of the
    // grid's extent, 2 <= L <= 7 (R-12b), by the oracle's exact power-of-two comparisons
    int lnear = 2;
    while (lnear < 7 && BA > ldexp(P.grid_extent, lnear - 3)) ++lnear;
    const int lev0 = UNIT ? P.split_level
                          : pred ? 0
                          : P.n_root == 1 ? 0
                          : j == 0 ? lnear
                          : P.n_root == 4 ? 2 : 1;
    int lev = lev0;
    const int rlev = UNIT ? P.split_level : 0;  // the walk ends when it climbs back here
    long long ix = UNIT ? (long long)(ukey & ((1ULL << kUnitShift) - 1)) : 0;
    for (;;) {
      const double p2 = __hiloint2double((1023 - lev) << 20, 0);  // 2^-lev, exact
      const double fa = (double)ix * p2, fb = (double)(ix + 1) * p2;
      const double a = __dadd_rn(A, __dmul_rn(BA, fa)), b = __dadd_rn(A, __dmul_rn(BA, fb));
      const double m = __dmul_rn(0.5, __dadd_rn(a, b)), hw = __dmul_rn(0.5, __dsub_rn(b, a));
      // ---- node phase: lanes 0..14 build the r' nodes of the GK15 rule
      int cnt = 0, skip = 0;
      bool full = false;
      const int nn = P.rule == RP_RULE_SIMPSON ? 5 : 15;  // r' nodes per segment
      if (lane < nn) {
        const int i = lane < 7 ? lane : (lane == 7 ? 7 : 14 - lane);
        double r;
        if (P.rule == RP_RULE_SIMPSON) {  // r_0 = a, r_2 = m, r_4 = b, r_1, r_3 midpoints
          r = lane == 0 ? a : lane == 2 ? m : lane == 4 ? b
                                : __dmul_rn(0.5, __dadd_rn(lane == 1 ? a : m, lane == 1 ? m : b));
        } else if (lane < 7) r = __dsub_rn(m, __dmul_rn(hw, c_xgk[i]));
        else if (lane == 7) r = m;
        else r = __dadd_rn(m, __dmul_rn(hw, c_xgk[i]));
        double cu, cv, w0, w1, w2;
        centre_at(it, P, r, cu, cv, w0, w1, w2);
        // arcs written straight into the warp's shared block (no local-memory staging)
        int na = arcs<KIND>(it, P, cu, cv, r, S.th1[lane], S.dth[lane]);
        NodeRec nr;
        nr.r = r; nr.cu = cu; nr.cv = cv; nr.w0 = w0; nr.w1 = w1; nr.w2 = w2;
        if (P.rule == RP_RULE_SIMPSON) {  // Boole h/90 (7,32,12,32,7); Simpson h/12 (1,4,2,4,1)
          const double h = __dsub_rn(b, a);
          nr.wk = h / 90.0 * (lane == 2 ? 12.0 : (lane & 1) ? 32.0 : 7.0);
          nr.wg = h / 12.0 * (lane == 2 ? 2.0 : (lane & 1) ? 4.0 : 1.0);
        } else {
          nr.wk = hw * c_wgk[i];
          nr.wg = (i & 1) ? hw * c_wg[i >> 1] : 0.0;  // Gauss nodes are the odd i (i = 7 centre)
        }
        S.node[lane] = nr;
        S.na[lane] = na;
        cnt = na < 0 ? N : na * (N + 1);
        full = na < 0;
        if (KIND == RP_SRC_GRID && VAR >= 4 && na > 0) {  // interior nodes (R-24, R-25b)
          skip = 2 * na;
          cnt = na * (N - 1);
        }
      }
      // integrand nodes of the rules over the 15 r' nodes (E, including the skipped arc end
      // nodes) and the largest per-node slot count (rounds): two independent butterflies
      if (lane < 16) S.cnt[lane] = lane < 15 ? cnt : 0;
      int E = cnt + skip, emax = cnt, skipped = skip;
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) {
        E += __shfl_xor_sync(0xffffffffu, E, o);
        emax = max(emax, __shfl_xor_sync(0xffffffffu, emax, o));
        skipped += __shfl_xor_sync(0xffffffffu, skipped, o);
      }
      // r' nodes whose circle lies wholly inside the support (warp-uniform bit per node)
      const unsigned fullmask = __ballot_sync(0xffffffffu, lane < nn && full);
      __syncwarp();
      // ---- evaluation phase
      double k0 = 0.0, k1 = 0.0, k2 = 0.0, g0 = 0.0, g1 = 0.0, g2 = 0.0;
      // Lane <-> theta slot: rounds of 32 slots, each lane running all 15 r' nodes of its slot
      // with the register stencil cache.  The round order alternates from segment to segment,
      // so the first round of a segment finds the cell left by the last round of the previous
      // (radially adjacent) segment.  Grid path: whole rounds (arc end nodes skipped, R-24: at
      // most 2 idle slots per arc); analytic sources: full rounds, then the leftover slots of
      // 65-node arcs as (slot, node) units.
      // r' nodes that carry a G7 (or Simpson) weight: all five Simpson nodes, else the odd GK15
      // nodes (the Gauss nodes; warp-uniform, kept in a register instead of re-reading P.rule)
      const unsigned gmask = P.rule == RP_RULE_SIMPSON ? 0x1Fu : 0x2AAAu;
      const int rounds = (KIND == RP_SRC_GRID && VAR >= 4) ? (emax + 31) >> 5 : emax >> 5;
      const int left = (KIND == RP_SRC_GRID && VAR >= 4) ? 0 : emax - 32 * rounds;
      if (KIND == RP_SRC_GRID && VAR >= 4) {
        for (int rr = 0; rr < rounds; ++rr) {
          const int r = (nseg & 1) ? rounds - 1 - rr : rr;
          pipelined_round<(VAR == 6 || VAR == 7)>(it, P, S, trig_full, 32 * r + lane, nn, N, wfull, third, st,
                                    ccell, k0, k1, k2, g0, g1, g2, fullmask, gmask);
        }
      } else {
        for (int rr = 0; rr < rounds; ++rr) {
          const int r = (nseg & 1) ? rounds - 1 - rr : rr;
          eval_nodes<KIND>(it, P, S, trig_full, 32 * r + lane, 0, nn, N, wfull, third, k0, k1,
                           k2, g0, g1, g2);
        }
      }
      for (int u = lane; u < nn * left; u += 32) {
        const int e = 32 * rounds + u / nn, n = u - nn * (u / nn);
        eval_nodes<KIND>(it, P, S, trig_full, e, n, n + 1, N, wfull, third, k0, k1, k2, g0, g1,
                         g2);
      }
      k0 = warp_sum(k0); k1 = warp_sum(k1); k2 = warp_sum(k2);
      g0 = warp_sum(g0); g1 = warp_sum(g1); g2 = warp_sum(g2);
      __syncwarp();
      evals += (unsigned)E;
      nskip += (unsigned)skipped;
      ++nseg;
      if (lev > maxlev) maxlev = lev;
      double err = fabs(k0 - g0);
      err = fmax(err, fabs(k1 - g1));
      err = fmax(err, fabs(k2 - g2));
      const double tol = tol0 * p2;
      if (fabs(err - tol) < 1e-9 * tol) ++ties;
      bool finished = false;
      if (err <= tol || lev >= P.max_depth) {
        if (!(err <= tol)) ++capped;
        ++nleaf;
        if ((VAR == 5 || VAR == 7) && lane == 0) {  // the accepted partition, for P:104 next call
          const unsigned long long pos = atomicAdd(P.leaf_count, 1ULL);
          if (pos < (unsigned long long)P.leaf_cap)
            P.leaf_rec[pos] = make_double4(a, b, (double)item, 0.0);
        }
        s_phi += k0; s_ax += k1; s_ay += k2; s_err += err;
        finished = true;
      } else if (!UNIT && P.split_level > 0 && lev + 1 == P.split_level && j < P.split_j &&
                 ndef < P.unit_budget) {
        // defer both children as subtree units into the item's own slots, in DFS order (the
        // per-item budget is counted in that order: deterministic, and never full)
        if (lane == 0) {
          const unsigned long long base = (unsigned long long)item << kUnitShift;
          const size_t slot = ((size_t)p * P.split_j + j) * P.unit_budget + ndef;
          P.unit_key[slot] = base | (unsigned long long)(2 * ix);
          P.unit_key[slot + 1] = base | (unsigned long long)(2 * ix + 1);
        }
        ndef += 2;
        finished = true;
      }
      if (finished) {
        while ((ix & 1) && lev > rlev) { ix >>= 1; --lev; }
        if (lev == rlev) {
          if (UNIT || !pred) break;
          // next root interval of the merged partition, if any reaches into [A, B]
          bool more = false;
          for (; rt < rt_end && P.bp[rt] < ab.y; ++rt) {
            const double a = fmax(P.bp[rt], ab.x), b = fmin(P.bp[rt + 1], ab.y);
            if (a < b) {
              A = a; BA = __dsub_rn(b, a); ++rt; more = true;
              tol0 = __ddiv_rn(__dmul_rn(P.tau, BA), P.R);
              break;
            }
          }
          if (!more) break;
          ix = 0;
          continue;
        }
        ++ix;
        // levels above the roots are never evaluated: from a sibling there, go down to the
        // first root below it (quarters: after quarter 1, quarter 2)
        while (lev < lev0) { ++lev; ix <<= 1; }
      } else {
        ++lev;
        ix <<= 1;
      }
    }
    if (lane == 0) {
      const size_t o = UNIT ? (size_t)uidx : (size_t)item;
      (UNIT ? P.unit_val : item_val)[o] = make_double4(s_phi, s_ax, s_ay, s_err);
      (UNIT ? P.unit_cnt : item_cnt)[o] = make_int4(nseg, nleaf, capped, ties);
      (UNIT ? P.unit_aux : item_aux)[o] = make_uint2((unsigned)maxlev, evals);
      if (nskip) atomicAdd(&counters[C_SKIP], (unsigned long long)nskip);
      if (!UNIT && P.split_level > 0 && j < P.split_j) {
        P.unit_ndef[(size_t)p * P.split_j + j] = ndef;
        if (ndef) atomicAdd(&counters[C_UNITS], (unsigned long long)ndef);
      }
    }
  }
}

// ------------------------------------------------------------- subtree units
__global__ void k_iota(int32_t* a, long long n) {
  const long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x;
  if (i < n) a[i] = (int32_t)i;
}

// Launch order of the units over all fixed slots (nslots = near-field items x unit_budget):
// a used slot gets its item's segment count of the previous step (the forecast), largest
// first (ties by slot); unused slots sort last.  The unit launch takes the first
// counters[C_UNITS] entries, so nothing is sized on the host.
__global__ void k_unit_order_keys(long long nslots, int budget, const int32_t* __restrict__ ndef,
                                  const unsigned long long* __restrict__ key,
                                  const uint16_t* __restrict__ cost,
                                  unsigned long long* __restrict__ okey) {
  const long long s = blockIdx.x * (long long)blockDim.x + threadIdx.x;
  if (s >= nslots) return;
  if ((int)(s % budget) >= ndef[s / budget]) {
    okey[s] = ~0ULL;
    return;
  }
  const unsigned long long item = key[s] >> kUnitShift;
  okey[s] = ((unsigned long long)(0xFFFFu - cost[item]) << 32) | (unsigned long long)s;
}

// Add every near-field item's units to its own partial result, in slot (= DFS, = subtree
// index) order: one thread per item, so the sums are deterministic for any launch order.
__global__ void k_merge_units(int n_nf, int split_j, int kmax, int budget,
                              const int32_t* __restrict__ ndef, const double4* __restrict__ uv,
                              const int4* __restrict__ uc, const uint2* __restrict__ ua,
                              double4* __restrict__ item_val, int4* __restrict__ item_cnt,
                              uint2* __restrict__ item_aux) {
  const int f = blockIdx.x * blockDim.x + threadIdx.x;
  if (f >= n_nf) return;
  const int nd = ndef[f];
  if (nd == 0) return;
  const size_t it = (size_t)(f / split_j) * kmax + (f % split_j);
  double4 v = item_val[it];
  int4 c = item_cnt[it];
  uint2 a = item_aux[it];
  for (int k = 0; k < nd; ++k) {
    const size_t u = (size_t)f * budget + k;
    const double4 w = uv[u];
    const int4 d = uc[u];
    const uint2 b = ua[u];
    v.x += w.x; v.y += w.y; v.z += w.z; v.w += w.w;
    c.x += d.x; c.y += d.y; c.z += d.z; c.w += d.w;
    a.x = max(a.x, b.x);
    a.y += b.y;
  }
  item_val[it] = v;
  item_cnt[it] = c;
  item_aux[it] = a;
}

// ------------------------------------------------------------- k_reduce
__global__ void k_reduce(int npts, int kmax, int kap, const uint32_t* __restrict__ key,
                         const double4* __restrict__ val, const int4* __restrict__ cnt,
                         const uint2* __restrict__ aux, const int32_t* __restrict__ owner,
                         int rank, const int32_t* __restrict__ row_of, int world,
                         double* __restrict__ phi, double* __restrict__ ax,
                         double* __restrict__ ay, double* __restrict__ err,
                         int32_t* __restrict__ nseg, double* __restrict__ shard,
                         uint16_t* __restrict__ cost, int32_t* __restrict__ nseg_pt,
                         uint16_t* __restrict__ leaves, int2* __restrict__ point_cnt,
                         unsigned long long* __restrict__ counters) {
  int p = blockIdx.x * blockDim.x + threadIdx.x;
  if (p >= npts) return;
  if (owner && owner[p] != rank) return;
  double a = 0.0, b = 0.0, c = 0.0, e = 0.0;
  long long ns = 0, nl = 0, cp = 0, ti = 0, ev = 0;
  int ml = 0;
  for (int j = 0; j < kmax; ++j) {
    size_t id = (size_t)p * kmax + j;
    if (j >= kap || key[id] == kEmptyKey) {
      cost[id] = 0;
      leaves[id] = 0;
      continue;
    }
    double4 v = val[id];
    int4 q = cnt[id];
    uint2 x = aux[id];
    a += v.x; b += v.y; c += v.z; e += v.w;
    ns += q.x; nl += q.y; cp += q.z; ti += q.w;
    ev += x.y;
    if ((int)x.x > ml) ml = (int)x.x;
    cost[id] = (uint16_t)(q.x < 0xFFFE ? q.x : 0xFFFE);
    leaves[id] = (uint16_t)(q.y < 0xFFFF ? q.y : 0xFFFF);  // observed access pattern n_j(p)
  }
  point_cnt[p] = make_int2((int)nl, (int)cp);  // per-point leaves / capped (rp_debug_point_counts)
  if (shard) {
    double* r = shard + 6 * (size_t)row_of[p];
    r[0] = (double)p; r[1] = a; r[2] = b; r[3] = c; r[4] = e; r[5] = (double)ns;
  } else {
    phi[p] = a;
    ax[p] = b;
    ay[p] = c;
    if (err) err[p] = e;
    if (nseg) nseg[p] = (int32_t)ns;
    nseg_pt[p] = (int32_t)ns;
  }
  atomicAdd(&counters[C_SEGS], (unsigned long long)ns);
  atomicAdd(&counters[C_LEAVES], (unsigned long long)nl);
  atomicAdd(&counters[C_CAPPED], (unsigned long long)cp);
  atomicAdd(&counters[C_TIES], (unsigned long long)ti);
  atomicAdd(&counters[C_EVALS], (unsigned long long)ev);
  atomicMax(&counters[C_MAXLEV], (unsigned long long)ml);
  atomicAdd(&counters[C_NOUT], 1ULL);
}

// ------------------------------------------------------------- shard map
__global__ void k_point_keys(int npts, const int32_t* __restrict__ nseg_pt, int have,
                             int32_t* __restrict__ key, int32_t* __restrict__ idx) {
  int p = blockIdx.x * blockDim.x + threadIdx.x;
  if (p >= npts) return;
  int w = have ? nseg_pt[p] : 0;
  key[p] = 0x7fffffff - (w < 0 ? 0 : w);  // ascending key = descending predicted work
  idx[p] = p;
}

__global__ void k_owner(int npts, int world, const int32_t* __restrict__ order,
                        int32_t* __restrict__ owner, int32_t* __restrict__ row) {
  int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= npts) return;
  int b = i / world, r = i % world;
  int rank = (b & 1) ? world - 1 - r : r;  // snake deal: longest-first, balanced
  int p = order[i];
  owner[p] = rank;
  row[p] = b;
}

__global__ void k_scatter(int npts, int world, int64_t cap, const double* __restrict__ sh,
                          double* __restrict__ phi, double* __restrict__ ax,
                          double* __restrict__ ay, double* __restrict__ err,
                          int32_t* __restrict__ nseg, int32_t* __restrict__ nseg_pt) {
  int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (t >= (int64_t)world * cap) return;
  int r = (int)(t / cap);
  int64_t b = t % cap;
  int64_t i = b * world + ((b & 1) ? world - 1 - r : r);
  if (i >= npts) return;
  const double* rec = sh + 6 * t;
  int p = (int)rec[0];
  phi[p] = rec[1];
  ax[p] = rec[2];
  ay[p] = rec[3];
  if (err) err[p] = rec[4];
  int ns = (int)rec[5];
  if (nseg) nseg[p] = ns;
  nseg_pt[p] = ns;
}

}  // namespace

int rp_alloc_potential_scratch(rp_ctx* ctx) {
  const rp_config& c = ctx->cfg;
  size_t npts = (size_t)c.nx * c.ny, nd = npts * c.history_depth;
  RP_CUDA(cudaMalloc(&ctx->clipAB, nd * sizeof(double2)));
  RP_CUDA(cudaMalloc(&ctx->sched_key, nd * sizeof(uint32_t)));
  RP_CUDA(cudaMalloc(&ctx->sched_key_sorted, nd * sizeof(uint32_t)));
  RP_CUDA(cudaMalloc(&ctx->sched_idx, nd * sizeof(int32_t)));
  RP_CUDA(cudaMalloc(&ctx->sched_order, nd * sizeof(int32_t)));
  RP_CUDA(cudaMalloc(&ctx->cost_prev, nd * sizeof(uint16_t)));
  RP_CUDA(cudaMalloc(&ctx->leaves_prev, nd * sizeof(uint16_t)));
  RP_CUDA(cudaMemset(ctx->leaves_prev, 0, nd * sizeof(uint16_t)));
  RP_CUDA(cudaMalloc(&ctx->cluster_dev, npts * sizeof(int32_t)));
  {
    // subtree work units: fixed slots, unit_budget per near-field item (item-major), so the
    // unit launch, its order sort and the merge are sized without a host round trip
    const long long nf = (long long)npts * ctx->split_j, slots = nf * kUnitBudget;
    ctx->unit_slots = slots;
    RP_CUDA(cudaMalloc(&ctx->unit_ndef, nf * sizeof(int32_t)));
    RP_CUDA(cudaMemset(ctx->unit_ndef, 0, nf * sizeof(int32_t)));
    RP_CUDA(cudaMalloc(&ctx->unit_key, slots * sizeof(unsigned long long)));
    RP_CUDA(cudaMalloc(&ctx->unit_okey, slots * sizeof(unsigned long long)));
    RP_CUDA(cudaMalloc(&ctx->unit_okey_sorted, slots * sizeof(unsigned long long)));
    RP_CUDA(cudaMalloc(&ctx->unit_iota, slots * sizeof(int32_t)));
    RP_CUDA(cudaMalloc(&ctx->unit_perm, slots * sizeof(int32_t)));
    RP_CUDA(cudaMalloc(&ctx->unit_val, slots * sizeof(double4)));
    RP_CUDA(cudaMalloc(&ctx->unit_cnt, slots * sizeof(int4)));
    RP_CUDA(cudaMalloc(&ctx->unit_aux, slots * sizeof(uint2)));
    k_iota<<<(unsigned)((slots + 255) / 256), 256>>>(ctx->unit_iota, slots);
    RP_CUDA(cudaGetLastError());
  }
  RP_CUDA(cudaMemset(ctx->cost_prev, 0, nd * sizeof(uint16_t)));
  RP_CUDA(cudaMalloc(&ctx->item_val, nd * sizeof(double4)));
  RP_CUDA(cudaMalloc(&ctx->item_cnt, nd * sizeof(int4)));
  RP_CUDA(cudaMalloc(&ctx->item_aux, nd * sizeof(uint2)));
  RP_CUDA(cudaMalloc(&ctx->counters, 16 * sizeof(unsigned long long)));
  RP_CUDA(cudaMalloc(&ctx->amp_dev, ctx->H * sizeof(double)));
  RP_CUDA(cudaMalloc(&ctx->point_key, npts * sizeof(int32_t)));
  RP_CUDA(cudaMalloc(&ctx->point_key_sorted, npts * sizeof(int32_t)));
  RP_CUDA(cudaMalloc(&ctx->point_idx, npts * sizeof(int32_t)));
  RP_CUDA(cudaMalloc(&ctx->point_order, npts * sizeof(int32_t)));
  RP_CUDA(cudaMalloc(&ctx->point_owner, npts * sizeof(int32_t)));
  RP_CUDA(cudaMalloc(&ctx->nseg_prev_pt, npts * sizeof(int32_t)));
  RP_CUDA(cudaMalloc(&ctx->point_cnt, npts * sizeof(int2)));
  RP_CUDA(cudaMemset(ctx->point_cnt, 0, npts * sizeof(int2)));
  RP_CUDA(cudaMemset(ctx->nseg_prev_pt, 0, npts * sizeof(int32_t)));
  // full-circle trapezoid nodes (cos, sin)(m * 2 pi / N), R-11
  double2* h = new double2[c.n_theta];
  for (int m = 0; m < c.n_theta; ++m) {
    double th = (double)m * (2.0 * M_PI / c.n_theta);
    h[m] = make_double2(cos(th), sin(th));
  }
  cudaError_t e = cudaMalloc(&ctx->trig_full, c.n_theta * sizeof(double2));
  if (e == cudaSuccess) e = cudaMemcpy(ctx->trig_full, h, c.n_theta * sizeof(double2), cudaMemcpyHostToDevice);
  delete[] h;
  RP_CUDA(e);
  return RP_OK;
}

template <int KIND, int VAR, bool UNIT = false>
static int launch_integrate_one(rp_ctx* ctx, const Params& P) {
  // persistent grid: resident warps per SM x SMs (occupancy queried once per instantiation)
  static int occ_of_dev[64] = {0};
  int& occ = occ_of_dev[ctx->cfg.device & 63];
  const size_t smem = 0;  // the warp's block is a static __shared__ variable
  if (occ == 0) {
    RP_CUDA(cudaFuncSetAttribute(k_integrate<KIND, VAR, UNIT>,
                                 cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    int o = 0;
    RP_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&o, k_integrate<KIND, VAR, UNIT>,
                                                          32 * kWarps, smem));
    occ = o < 1 ? 1 : o;
  }
  k_integrate<KIND, VAR, UNIT><<<ctx->sm_count * occ, 32 * kWarps, smem, ctx->stream>>>(
      P, ctx->sched_order, ctx->clipAB, ctx->trig_full, ctx->item_val, ctx->item_cnt,
      ctx->item_aux, ctx->counters);
  RP_CHECK_LAUNCH();
  return RP_OK;
}

// The integrator: the items, then (split_level > 0) the deferred subtree units and their
// merge into the items.  One profiling record covers the whole integration.  Everything is
// stream-ordered: the unit launch reads its count from the device (no host synchronisation).
template <int KIND, int VAR>
static int launch_integrate(rp_ctx* ctx, const Params& P) {
  ProfScope ps(ctx, PK_INTEGRATE);
  cudaStream_t st = ctx->stream;
  const bool split = KIND == RP_SRC_GRID && VAR >= 4 && P.split_level > 0;
  const long long nf = (long long)P.npts * P.split_j;
  if (split) RP_CUDA(cudaMemsetAsync(ctx->unit_ndef, 0, nf * sizeof(int32_t), st));
  int rc = launch_integrate_one<KIND, VAR, false>(ctx, P);
  if (rc || !split) return rc;
  ProfScope pu(ctx, PK_UNITS);
  const long long slots = nf * P.unit_budget;
  k_unit_order_keys<<<(unsigned)((slots + 255) / 256), 256, 0, st>>>(
      slots, P.unit_budget, ctx->unit_ndef, ctx->unit_key, ctx->cost_prev, ctx->unit_okey);
  RP_CHECK_LAUNCH();
  size_t tmp = 0;
  RP_CUDA(cub::DeviceRadixSort::SortPairs(nullptr, tmp, ctx->unit_okey, ctx->unit_okey_sorted,
                                          ctx->unit_iota, ctx->unit_perm, (int)slots, 0, 48, st));
  rc = rp_ensure_cub_tmp(ctx, tmp);
  if (rc) return rc;
  tmp = ctx->cub_tmp_bytes;
  RP_CUDA(cub::DeviceRadixSort::SortPairs(ctx->cub_tmp, tmp, ctx->unit_okey, ctx->unit_okey_sorted,
                                          ctx->unit_iota, ctx->unit_perm, (int)slots, 0, 48, st));
  Params PU = P;
  PU.unit_order = ctx->unit_perm;
  rc = launch_integrate_one<KIND, VAR, true>(ctx, PU);
  if (rc) return rc;
  k_merge_units<<<(unsigned)((nf + 255) / 256), 256, 0, st>>>(
      (int)nf, P.split_j, P.kmax, P.unit_budget, ctx->unit_ndef, ctx->unit_val, ctx->unit_cnt,
      ctx->unit_aux, ctx->item_val, ctx->item_cnt, ctx->item_aux);
  RP_CHECK_LAUNCH();
  return RP_OK;
}

template <int KIND>
static int run_potentials(rp_ctx* ctx, Params P, int32_t rank, int32_t world,
                          double* phi, double* ax, double* ay, double* err, int32_t* nseg,
                          double* shard_out, int64_t cap) {
  cudaStream_t st = ctx->stream;
  const int64_t nd = (int64_t)P.npts * P.kmax;
  const int32_t* owner = nullptr;
  int32_t* row = nullptr;
  if (shard_out) {
    // shard map from the previous step's per-point counts (identical on every rank)
    k_point_keys<<<(P.npts + 255) / 256, 256, 0, st>>>(P.npts, ctx->nseg_prev_pt,
                                                        ctx->has_forecast, ctx->point_key,
                                                        ctx->point_idx);
    RP_CHECK_LAUNCH();
    size_t tmp = 0;
    RP_CUDA(cub::DeviceRadixSort::SortPairs(nullptr, tmp, ctx->point_key, ctx->point_key_sorted,
                                            ctx->point_idx, ctx->point_order, P.npts, 0, 32, st));
    int rc = rp_ensure_cub_tmp(ctx, tmp);
    if (rc) return rc;
    tmp = ctx->cub_tmp_bytes;
    RP_CUDA(cub::DeviceRadixSort::SortPairs(ctx->cub_tmp, tmp, ctx->point_key,
                                            ctx->point_key_sorted, ctx->point_idx,
                                            ctx->point_order, P.npts, 0, 32, st));
    k_owner<<<(P.npts + 255) / 256, 256, 0, st>>>(P.npts, world, ctx->point_order,
                                                   ctx->point_owner, ctx->point_key);
    RP_CHECK_LAUNCH();
    owner = ctx->point_owner;
    row = ctx->point_key;  // reused as row index
    RP_CUDA(cudaMemsetAsync(shard_out, 0, (size_t)cap * 6 * sizeof(double), st));
  }
  RP_CUDA(cudaMemsetAsync(ctx->counters, 0, 16 * sizeof(unsigned long long), st));
  if (nd > 0) {
    {
      ProfScope ps(ctx, PK_CLIP);
      k_clip<KIND><<<(unsigned)((nd + 255) / 256), 256, 0, st>>>(
          P, owner, rank,
          (ctx->has_forecast && ctx->sched_policy != RP_SCHED_INDEX) ? ctx->cost_prev : nullptr,
          ctx->sched_policy, ctx->sched_k, ctx->clipAB,
          ctx->sched_key, ctx->sched_idx, ctx->counters);
      RP_CHECK_LAUNCH();
    }
    {
      ProfScope ps(ctx, PK_SORT);
      const int kbits = ctx->sched_policy == RP_SCHED_SUBREGION ? 32 : 16;
      size_t tmp = 0;
      RP_CUDA(cub::DeviceRadixSort::SortPairs(nullptr, tmp, ctx->sched_key, ctx->sched_key_sorted,
                                              ctx->sched_idx, ctx->sched_order, (int)nd, 0, kbits, st));
      int rc = rp_ensure_cub_tmp(ctx, tmp);
      if (rc) return rc;
      tmp = ctx->cub_tmp_bytes;
      RP_CUDA(cub::DeviceRadixSort::SortPairs(ctx->cub_tmp, tmp, ctx->sched_key,
                                              ctx->sched_key_sorted, ctx->sched_idx,
                                              ctx->sched_order, (int)nd, 0, kbits, st));
    }
    const int var = KIND != RP_SRC_GRID ? 0 : (P.interp == RP_INTERP_LAGRANGE3 ? 6 : 4);
    ctx->pred_info.active = 0;
    if (KIND == RP_SRC_GRID && ctx->pred_on && ctx->have_leaves && !shard_out && var != 0) {
      // Predictive-RP lines 1-12 on the host (R-26): forecast, partition, cluster, merge
      int rc = rp_predictive_setup(ctx, P.kap);
      if (rc) return rc;
      P.bp = ctx->bp_dev;
      P.bp_off = ctx->bp_off_dev;
      P.cluster = ctx->cluster_dev;
    }
    const bool rec = KIND == RP_SRC_GRID && ctx->pred_on && ctx->pred_part == RP_PART_ADAPTIVE &&
                     !shard_out && var != 0 && ctx->leaf_rec;
    if (rec) {  // this call's accepted leaves, for the next call's adaptive partitioning
      RP_CUDA(cudaMemsetAsync(ctx->leaf_count_dev, 0, sizeof(unsigned long long), st));
      P.leaf_rec = ctx->leaf_rec;
      P.leaf_count = ctx->leaf_count_dev;
      P.leaf_cap = ctx->leaf_cap;
    }
    ctx->leaf_valid = rec ? 1 : 0;
    P.split_level = (KIND == RP_SRC_GRID && var >= 4 && P.bp_off == nullptr) ? ctx->split_level : 0;
    P.split_j = ctx->split_j;
    P.unit_budget = ctx->unit_budget;  // <= kUnitBudget, the slots allocated per item
    P.unit_ndef = ctx->unit_ndef;
    P.unit_key = ctx->unit_key;
    P.unit_val = ctx->unit_val;
    P.unit_cnt = ctx->unit_cnt;
    P.unit_aux = ctx->unit_aux;
    int rc2 = KIND != RP_SRC_GRID ? launch_integrate<KIND, 0>(ctx, P)
              : var == 6 ? (P.leaf_rec ? launch_integrate<KIND, kGridVar + 3>(ctx, P)
                                         : launch_integrate<KIND, kGridVar + 2>(ctx, P))
              : P.leaf_rec ? launch_integrate<KIND, kGridVar + 1>(ctx, P)
                           : launch_integrate<KIND, kGridVar>(ctx, P);
    if (rc2) return rc2;
  }
  ProfScope ps_red(ctx, PK_REDUCE);
  k_reduce<<<(P.npts + 255) / 256, 256, 0, st>>>(
      P.npts, P.kmax, P.kap, ctx->sched_key, ctx->item_val, ctx->item_cnt, ctx->item_aux, owner,
      rank, row, world, phi, ax, ay, err, nseg, shard_out, ctx->cost_prev, ctx->nseg_prev_pt,
      ctx->leaves_prev, ctx->point_cnt, ctx->counters);
  RP_CHECK_LAUNCH();
  ctx->has_forecast = 1;
  ctx->have_leaves = shard_out ? 0 : 1;
  return RP_OK;
}

int rp_potentials_impl(rp_ctx* ctx, int kind, const double src[6], int32_t rank, int32_t world,
                       double* phi, double* ax, double* ay, double* err, int32_t* nseg,
                       double* shard_out, int64_t cap, int64_t* n_out, rp_potential_info* info) {
  const rp_config& c = ctx->cfg;
  if (ctx->k < 0) return rp_fail(ctx, RP_ESTATE, "potentials before the first deposit");
  if (!shard_out && (!phi || !ax || !ay)) return rp_fail(ctx, RP_EINVAL, "potentials: null output");
  Params P;
  P.nx = c.nx; P.ny = c.ny; P.PX = ctx->PX; P.npts = c.nx * c.ny; P.kmax = c.history_depth;
  P.kap = kappa_of(ctx); P.k = ctx->k; P.H = ctx->H; P.n_theta = c.n_theta;
  P.max_depth = c.max_depth; P.n_root = c.n_root; P.rule = c.outer_rule;
  P.inv_n_theta = (c.n_theta & (c.n_theta - 1)) == 0 ? 1.0 / (double)c.n_theta : 0.0;
  P.grid_extent = std::max(c.nx * c.hx, c.ny * c.hy);
  P.variant = 0;
  P.interp = c.interp;
  P.hx = c.hx; P.hy = c.hy; P.inv_hx = 1.0 / c.hx; P.inv_hy = 1.0 / c.hy;
  P.cdt = c.c * c.dt; P.tau = c.tau; P.R = (double)P.kap * P.cdt;
  P.slot_doubles = ctx->slot_doubles; P.ring = ctx->ring; P.frames = ctx->frames_dev;
  P.amp = ctx->amp_dev;
  P.bp = nullptr; P.bp_off = nullptr; P.cluster = nullptr;
  P.leaf_rec = nullptr; P.leaf_count = nullptr; P.leaf_cap = 0;
  P.split_level = 0; P.split_j = 0; P.unit_budget = 0; P.unit_ndef = nullptr;
  P.unit_order = nullptr; P.unit_key = nullptr; P.unit_val = nullptr;
  P.unit_cnt = nullptr; P.unit_aux = nullptr;
  P.sx0 = src ? src[0] : 0; P.sy0 = src ? src[1] : 0; P.swidth = src ? src[2] : 0;
  P.sq = src ? src[3] : 0; P.sbx = src ? src[4] : 0; P.sby = src ? src[5] : 0;
  int rc;
  if (kind == RP_SRC_GRID)
    rc = run_potentials<RP_SRC_GRID>(ctx, P, rank, world, phi, ax, ay, err, nseg, shard_out, cap);
  else if (kind == RP_SRC_GAUSS)
    rc = run_potentials<RP_SRC_GAUSS>(ctx, P, rank, world, phi, ax, ay, err, nseg, shard_out, cap);
  else
    rc = run_potentials<RP_SRC_DISK>(ctx, P, rank, world, phi, ax, ay, err, nseg, shard_out, cap);
  if (rc) return rc;
  if (info || n_out) {
    unsigned long long h[16];
    RP_CUDA(cudaMemcpyAsync(h, ctx->counters, sizeof(h), cudaMemcpyDeviceToHost, ctx->stream));
    RP_CUDA(cudaStreamSynchronize(ctx->stream));
    if (info) {
      info->items = (int64_t)h[C_ITEMS];
      info->evals = (int64_t)h[C_EVALS];
      info->segments = (int64_t)h[C_SEGS];
      info->nodes = (c.outer_rule == RP_RULE_SIMPSON ? 5 : 15) * (int64_t)h[C_SEGS];
      info->leaves = (int64_t)h[C_LEAVES];
      info->capped = (int64_t)h[C_CAPPED];
      info->ties = (int64_t)h[C_TIES];
      info->max_level = (int32_t)h[C_MAXLEV];
      info->kappa = P.kap;
      info->skipped = (int64_t)h[C_SKIP];
      info->units = (int64_t)h[C_UNITS];
    }
    if (n_out) *n_out = (int64_t)h[C_NOUT];
  }
  return RP_OK;
}

int rp_scatter_impl(rp_ctx* ctx, const double* shards, int32_t world, int64_t cap, double* phi,
                    double* ax, double* ay, double* err, int32_t* nseg) {
  const rp_config& c = ctx->cfg;
  int npts = c.nx * c.ny;
  int64_t tot = (int64_t)world * cap;
  k_scatter<<<(unsigned)((tot + 255) / 256), 256, 0, ctx->stream>>>(npts, world, cap, shards, phi,
                                                                     ax, ay, err, nseg,
                                                                     ctx->nseg_prev_pt);
  RP_CHECK_LAUNCH();
  ctx->has_forecast = 1;
  return RP_OK;
}
