/*
 * rp_oracle.c -- CPU ORACLE for the retarded-potential step of
 *   Arumugam, Godunov, Islam, Ranjan, Terzic, Zubair,
 *   "A Machine Learning Approach for Efficient Parallel Simulation of Beam
 *    Dynamics on GPUs", ICPP'17  (PAPER.md = /root/reference/PAPER.md).
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and the
 * cpu_baseline / --impl reference legs of bench.py may load this library.
 * The product path (paper_conf_icpp_arumugamrztgi17_b200/) never links,
 * imports or calls it, and this file includes nothing from the product.
 *
 * Plain, slow, obviously-correct FP64.  Compiled with -O2 -ffp-contract=off
 * (no FMA contraction), one OpenMP "parallel for schedule(dynamic)" over mesh
 * points and nothing else clever.  Every function cites the PAPER.md line
 * (P:NN) it follows, or the DESIGN.md "reading" (R-n) that fills a gap in the
 * paper (the paper's integral limits, inner rule and stencil live in its
 * absent references [9], [14]).
 *
 * Pins (tests/test_oracle_*.py, -m "not gpu"): GK15 monomial exactness,
 * TSC / Lagrange weight identities, arcs vs dense theta sampling, clip vs a
 * brute r' scan, Gaussian and uniform-disk closed forms (static and with a
 * quadratic-in-time amplitude), brute-force Gauss-Legendre outer integral,
 * Cartesian fine-cell sum, deposit charge conservation and J = rho*beta,
 * (M, tau) -> (2M, 2tau) scaling, J = 0 => A = 0, FD exactness on
 * quadratics, Boris |u| conservation and gyration radius, steady-state
 * stationarity in the bend.
 * "parity unpinned": none of the exported functions.
 */
#include <float.h>
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

/* R-28: a decision within this many ulp of |K_rho| + |G_rho| is flagged (noise_ties) */
#define ORC_NOISE_TIE 4.0

#ifndef M_PI
#define M_PI 3.14159265358979323846
#endif

/* ------------------------------------------------------------------ */
/* Types (mirrored by oracle/__init__.py with ctypes)                  */
/* ------------------------------------------------------------------ */
typedef struct { double ox, oy, c, s; } orc_frame; /* lab = O + u(c,s) + v(-s,c) */

typedef struct {
  int32_t nx, ny;
  double hx, hy;
  double c, dt;      /* subregion width c*dt                         */
  double tau;        /* absolute tolerance per component (1e-6)      */
  int32_t n_theta;   /* inner panels per arc (R-11)                          */
  int32_t max_depth; /* bisection cap (R-12)                                 */
  int32_t n_root;    /* 2: both halves of [A,B] (quarters in S_0); 1: [A,B]; 4: quarters */
  int32_t kappa_max; /* history depth (R-4)                                  */
  int32_t rule;      /* outer segment rule: 0 = GK15 (R-8), 1 = Simpson/Boole (R-22) */
  int32_t interp;    /* spatial weights: 0 = TSC (R-6), 1 = quadratic Lagrange (R-25)  */
} orc_params;

typedef struct {
  const double* ring;      /* [H][ny][nx][4]: rho, rho*beta_x, rho*beta_y, 0 */
  const orc_frame* frames; /* [H]                                            */
  int32_t H;               /* ring slots = kappa_max + 2                      */
  int32_t k;               /* current step                                    */
  int32_t n_pre;           /* number of pre-history levels l = -1..-n_pre     */
} orc_hist;

enum { ORC_SRC_GRID = 0, ORC_SRC_GAUSS = 1, ORC_SRC_DISK = 2 };
typedef struct {
  int32_t kind;       /* ORC_SRC_*                                                */
  double x0, y0;      /* analytic source centre, frame-local coordinates          */
  double width;       /* gauss: sigma ; disk: radius a                           */
  double q;           /* gauss: total charge Q ; disk: surface density sigma_s   */
  double bx, by;      /* analytic source: beta (current = rho * beta)            */
  const double* amp;  /* analytic source: amplitude per ring slot [H] (NULL = 1)  */
} orc_source;

typedef struct {
  double phi, ax, ay, err;      /* I_rho, I_{rho bx}, I_{rho by}, sum of leaf errors */
  int32_t nseg, nleaf, capped, ties, max_level;
  int32_t noise_ties;           /* decisions inside the rounding noise of err (R-28)  */
  int64_t evals;                /* integrand evaluations (flop census)                */
  int64_t nodes;                /* r' nodes evaluated (15 per segment)                */
  double min_margin;            /* min |err - tol| / tol over all decisions           */
  int64_t chase_segs;           /* diagnostics: segments whose subtree ends in a */
  int64_t chase_evals;          /* capped leaf, and their integrand evaluations          */
  double min_noise;             /* min |err - tol| / (eps (|K_rho| + |G_rho|)) (R-28)   */
} orc_result;

/* ------------------------------------------------------------------ */
/* GK15 constants (QUADPACK qk15), the outer rule of R-8               */
/* ------------------------------------------------------------------ */
static const double XGK[8] = {
    0.991455371120812639206854697526329, 0.949107912342758524526189684047851,
    0.864864423359769072789712788640926, 0.741531185599394439863864773280788,
    0.586087235467691130294144845693013, 0.405845151377397166906606412076961,
    0.207784955007898467600689403773245, 0.000000000000000000000000000000000};
static const double WGK[8] = {
    0.022935322010529224963732008058970, 0.063092092629978553290700663189204,
    0.104790010322250183839876322541518, 0.140653259715525918745189590510238,
    0.169004726639267902826583426598550, 0.190350578064785409913256402421014,
    0.204432940075298892414161999234649, 0.209482141084727828012999174891714};
/* Gauss-7 weights on XGK[1], XGK[3], XGK[5], XGK[7] */
static const double WG[4] = {
    0.129484966168869693270611432679082, 0.279705391489276667901467771423780,
    0.381830050505118944950369775488975, 0.417959183673469387755102040816327};

void orc_gk15_constants(double* xgk, double* wgk, double* wg) {
  for (int i = 0; i < 8; ++i) { xgk[i] = XGK[i]; wgk[i] = WGK[i]; }
  for (int i = 0; i < 4; ++i) wg[i] = WG[i];
}

/* ------------------------------------------------------------------ */
/* Weights                                                              */
/* ------------------------------------------------------------------ */
/* TSC (quadratic B-spline) weights for nodes -1, 0, +1 about the nearest
 * node at offset delta in [-1/2, 1/2] (R-6: the "27 neighbouring points" of
 * P:45 are 3x3 spatial TSC nodes x 3 time levels). */
void orc_tsc_weights(double d, double* w) {
  double a = 0.5 - d, b = 0.5 + d;
  w[0] = 0.5 * (a * a);
  w[1] = 0.75 - d * d;
  w[2] = 0.5 * (b * b);
}

/* Quadratic Lagrange weights in time for levels (l0,l1,l2) = (k-j-2,k-j-1,k-j)
 * at nodes tau = -1, 0, +1 (R-2). */
void orc_lagrange3_weights(double t, double* w) {
  w[0] = 0.5 * t * (t - 1.0);
  w[1] = 1.0 - t * t;
  w[2] = 0.5 * t * (t + 1.0);
}

/* ------------------------------------------------------------------ */
/* Binning and deposition (step 1 of the 4-step loop; R-14)       */
/* ------------------------------------------------------------------ */
static void to_local(const orc_frame* F, double x, double y, double* u, double* v) {
  double dx = x - F->ox, dy = y - F->oy;
  *u = F->c * dx + F->s * dy;
  *v = F->c * dy - F->s * dx;
}

/* Nearest-node bin (R-13: round half up).  Returns iy*nx+ix, or -1 when the
 * 3x3 stencil would leave the grid (particle lost). */
int32_t orc_bin_of(double x, double y, const orc_frame* F, double hx, double hy,
                   int32_t nx, int32_t ny, int32_t* ix_out, int32_t* iy_out,
                   double* dx_out, double* dy_out) {
  double u, v;
  to_local(F, x, y, &u, &v);
  double tx = u / hx, ty = v / hy;
  double fx = floor(tx + 0.5), fy = floor(ty + 0.5);
  double dx = tx - fx, dy = ty - fy;
  int32_t ok = (fx >= 1.0 && fx <= (double)(nx - 2) && fy >= 1.0 && fy <= (double)(ny - 2));
  int32_t ix = ok ? (int32_t)fx : -1, iy = ok ? (int32_t)fy : -1;
  if (ix_out) *ix_out = ix;
  if (iy_out) *iy_out = iy;
  if (dx_out) *dx_out = dx;
  if (dy_out) *dy_out = dy;
  return ok ? iy * nx + ix : -1;
}

/* TSC deposit of n particles (x, y, ux, uy with u = gamma*beta) of charge q
 * each onto M[ny][nx][4] (accumulated; caller zeroes).  Particle loop in
 * index order.  Returns the lost charge. */
double orc_deposit(int64_t n, const double* x, const double* y, const double* ux,
                   const double* uy, double q, const orc_frame* F, int32_t nx,
                   int32_t ny, double hx, double hy, double* M, int32_t* bins) {
  double q_lost = 0.0;
  for (int64_t i = 0; i < n; ++i) {
    int32_t ix, iy;
    double dx, dy;
    int32_t b = orc_bin_of(x[i], y[i], F, hx, hy, nx, ny, &ix, &iy, &dx, &dy);
    if (bins) bins[i] = b;
    if (b < 0) { q_lost += q; continue; }
    double g = sqrt(1.0 + ux[i] * ux[i] + uy[i] * uy[i]);
    double bx = ux[i] / g, by = uy[i] / g;
    double wx[3], wy[3];
    orc_tsc_weights(dx, wx);
    orc_tsc_weights(dy, wy);
    for (int bb = 0; bb < 3; ++bb)
      for (int aa = 0; aa < 3; ++aa) {
        double w = q * wx[aa] * wy[bb] / (hx * hy);
        double* m = M + 4 * ((int64_t)(iy + bb - 1) * nx + (ix + aa - 1));
        m[0] += w;
        m[1] += w * bx;
        m[2] += w * by;
      }
  }
  return q_lost;
}

/* Rigid steady-state pre-history level (SURVEY 8(d) steady state; DESIGN R-23): the same
 * comoving bunch as step 0, viewed in frame Fl.  rho is copied; the lab current is rotated
 * by the angle between the frames, psi_l - psi_0:
 *   cos(psi_l - psi_0) = c_l c_0 + s_l s_0,  sin(psi_l - psi_0) = s_l c_0 - c_l s_0,
 *   J_l = [[cos, -sin], [sin, cos]] J_0.
 * M0, Ml: [ny][nx][4]. */
void orc_rigid_level(const double* M0, const orc_frame* F0, const orc_frame* Fl, int32_t nx,
                     int32_t ny, double* Ml) {
  double cd = Fl->c * F0->c + Fl->s * F0->s;
  double sd = Fl->s * F0->c - Fl->c * F0->s;
  for (int64_t i = 0; i < (int64_t)nx * ny; ++i) {
    const double* m = M0 + 4 * i;
    double* o = Ml + 4 * i;
    o[0] = m[0];
    o[1] = cd * m[1] - sd * m[2];
    o[2] = sd * m[1] + cd * m[2];
    o[3] = m[3];
  }
}

/* ------------------------------------------------------------------ */
/* History access ("stored linearly"; ring of H slots)            */
/* ------------------------------------------------------------------ */
static int32_t slot_of(int32_t level, int32_t H) { return ((level % H) + H) % H; }

/* Frame at retarded time: quadratic Lagrange in time through the frames of
 * levels l0,l1,l2 (R-7), written as X1 + w0 (X0-X1) + w2 (X2-X1) so that a
 * static frame is returned exactly.  No renormalisation of (c, s). */
static orc_frame frame_at(const orc_frame* F0, const orc_frame* F1, const orc_frame* F2,
                          const double* w) {
  orc_frame r;
  r.ox = F1->ox + w[0] * (F0->ox - F1->ox) + w[2] * (F2->ox - F1->ox);
  r.oy = F1->oy + w[0] * (F0->oy - F1->oy) + w[2] * (F2->oy - F1->oy);
  r.c = F1->c + w[0] * (F0->c - F1->c) + w[2] * (F2->c - F1->c);
  r.s = F1->s + w[0] * (F0->s - F1->s) + w[2] * (F2->s - F1->s);
  return r;
}

/* ------------------------------------------------------------------ */
/* Per-subregion context                                                */
/* ------------------------------------------------------------------ */
typedef struct {
  const orc_params* P;
  const orc_hist* Hh;
  const orc_source* S;
  double px, py;          /* mesh point, lab                                  */
  int32_t j;              /* subregion index (S_j = [j c dt, (j+1) c dt])      */
  const orc_frame* F[3];  /* frames of levels l0, l1, l2                       */
  const double* G[3];     /* grids of levels l0, l1, l2                        */
  double amp[3];          /* analytic amplitudes of the 3 levels               */
  double U0, U1, V0, V1;  /* support rectangle (frame-local)                   */
  int64_t evals;
  double* ends;           /* nullable: accepted leaves' left ends, then the last  */
  int64_t nends;          /* right end (the item's partition; R-26b)       */
  double last_b;          /* right end of the last accepted leaf, as computed     */
} subctx;

/* tau_t(r') = (j+1) - r'/(c dt) in [0,1] on S_j (t' = k dt - r'/c). */
static double tau_of(const subctx* X, double r) {
  return (double)(X->j + 1) - r / (X->P->c * X->P->dt);
}

/* Local centre (c_u, c_v) of the circle about p at retarded time t'(r). */
static void centre_at(const subctx* X, double r, double* cu, double* cv, double* w) {
  orc_lagrange3_weights(tau_of(X, r), w);
  orc_frame f = frame_at(X->F[0], X->F[1], X->F[2], w);
  double dx = X->px - f.ox, dy = X->py - f.oy;
  *cu = f.c * dx + f.s * dy;
  *cv = -f.s * dx + f.c * dy;
}

/* squared distance from (cu,cv) to the support (0 inside), and squared
 * distance to its farthest point (R-5: the limits of P:43). */
static void support_dist2(const subctx* X, double cu, double cv, double* dmin2, double* dmax2) {
  if (X->S->kind == ORC_SRC_DISK) {
    double ex = cu - X->S->x0, ey = cv - X->S->y0;
    double s = sqrt(ex * ex + ey * ey), a = X->S->width;
    double lo = s - a > 0.0 ? s - a : 0.0, hi = s + a;
    *dmin2 = lo * lo;
    *dmax2 = hi * hi;
    return;
  }
  double ex = 0.0, ey = 0.0;
  if (cu < X->U0) ex = X->U0 - cu; else if (cu > X->U1) ex = cu - X->U1;
  if (cv < X->V0) ey = X->V0 - cv; else if (cv > X->V1) ey = cv - X->V1;
  *dmin2 = ex * ex + ey * ey;
  double fx = fabs(cu - X->U0) > fabs(cu - X->U1) ? fabs(cu - X->U0) : fabs(cu - X->U1);
  double fy = fabs(cv - X->V0) > fabs(cv - X->V1) ? fabs(cv - X->V0) : fabs(cv - X->V1);
  *dmax2 = fx * fx + fy * fy;
}

static void dists_at(const subctx* X, double r, double* dmin2, double* dmax2) {
  double cu, cv, w[3];
  centre_at(X, r, &cu, &cv, w);
  support_dist2(X, cu, cv, dmin2, dmax2);
}

/* Support clip of S_j (R-5): [A,B] = {r in S_j :
 * d_min(r) <= r <= d_max(r)}, by 64-step bisection on squares.  Returns 0
 * when the subregion has no support. */
int32_t orc_clip(const subctx* X, double a, double b, double* A, double* B) {
  double dmn, dmx;
  dists_at(X, b, &dmn, &dmx);
  if (dmn > b * b) return 0;
  dists_at(X, a, &dmn, &dmx);
  if (dmx < a * a) return 0;
  /* lower end */
  dists_at(X, a, &dmn, &dmx);
  if (dmn <= a * a) {
    *A = a;
  } else {
    double lo = a, hi = b;
    for (int it = 0; it < 64; ++it) {
      double m = 0.5 * (lo + hi);
      dists_at(X, m, &dmn, &dmx);
      if (dmn <= m * m) hi = m; else lo = m;
    }
    *A = hi;
  }
  /* upper end */
  dists_at(X, b, &dmn, &dmx);
  if (dmx >= b * b) {
    *B = b;
  } else {
    double lo = a, hi = b;
    for (int it = 0; it < 64; ++it) {
      double m = 0.5 * (lo + hi);
      dists_at(X, m, &dmn, &dmx);
      if (dmx >= m * m) lo = m; else hi = m;
    }
    *B = lo;
  }
  return (*A < *B) ? 1 : 0;
}

/* ------------------------------------------------------------------ */
/* Arcs of circle (cu,cv; r) inside a rectangle (R-5, C.3e)             */
/* ------------------------------------------------------------------ */
static int inside_rect(double u, double v, double U0, double U1, double V0, double V1) {
  return u >= U0 && u <= U1 && v >= V0 && v <= V1;
}

static int cmp_double(const void* a, const void* b) {
  double x = *(const double*)a, y = *(const double*)b;
  return (x > y) - (x < y);
}

/* Writes up to 8 arcs as pairs (t1, t2) with t1 < t2 (t2 may exceed 2 pi for
 * the wrap-around arc).  Returns the number of arcs, or -1 for the full
 * circle. */
int32_t orc_arcs_rect(double cu, double cv, double r, double U0, double U1, double V0,
                      double V1, double* arcs) {
  double t[8];
  int n = 0;
  const double twopi = 2.0 * M_PI;
  double E[2] = {U0, U1};
  for (int e = 0; e < 2; ++e) { /* vertical edges u = E[e] */
    double d = (E[e] - cu) / r;
    if (fabs(d) < 1.0) {
      double al = acos(d);
      double c1 = al, c2 = twopi - al;
      double v1 = cv + r * sin(c1), v2 = cv + r * sin(c2);
      if (v1 >= V0 && v1 <= V1) t[n++] = c1;
      if (v2 >= V0 && v2 <= V1) t[n++] = c2;
    }
  }
  double Fv[2] = {V0, V1};
  for (int e = 0; e < 2; ++e) { /* horizontal edges v = Fv[e] */
    double d = (Fv[e] - cv) / r;
    if (fabs(d) < 1.0) {
      double be = asin(d);
      double c1 = be < 0.0 ? be + twopi : be, c2 = M_PI - be;
      double u1 = cu + r * cos(c1), u2 = cu + r * cos(c2);
      if (u1 >= U0 && u1 <= U1) t[n++] = c1;
      if (u2 >= U0 && u2 <= U1) t[n++] = c2;
    }
  }
  if (n == 0) return inside_rect(cu + r, cv, U0, U1, V0, V1) ? -1 : 0;
  qsort(t, (size_t)n, sizeof(double), cmp_double);
  int m = 0; /* merge exact duplicates */
  for (int i = 0; i < n; ++i)
    if (m == 0 || t[i] != t[m - 1]) t[m++] = t[i];
  int na = 0;
  for (int i = 0; i < m; ++i) {
    double t1 = t[i], t2 = (i + 1 < m) ? t[i + 1] : t[0] + twopi;
    double mid = 0.5 * (t1 + t2);
    if (inside_rect(cu + r * cos(mid), cv + r * sin(mid), U0, U1, V0, V1)) {
      arcs[2 * na] = t1;
      arcs[2 * na + 1] = t2;
      ++na;
    }
  }
  return na;
}

/* Arc of circle (cu,cv; r) inside the disk (x0,y0; a).  Same return
 * convention as orc_arcs_rect (test-only analytic source, C.4). */
int32_t orc_arcs_disk(double cu, double cv, double r, double x0, double y0, double a,
                      double* arcs) {
  double ex = x0 - cu, ey = y0 - cv;
  double s = sqrt(ex * ex + ey * ey);
  if (s + r <= a) return -1;
  if (r >= s + a || s >= r + a) return 0;
  double ph = atan2(ey, ex);
  double al = acos((r * r + s * s - a * a) / (2.0 * r * s));
  arcs[0] = ph - al;
  arcs[1] = ph + al;
  return 1;
}

/* ------------------------------------------------------------------ */
/* Integrand f^(p)(r', theta', t') (R-1, R-6, R-7)                 */
/* ------------------------------------------------------------------ */
/* TSC interpolation of one level at frame-local (u,v); out-of-range nodes 0. */
static void grid_interp(const orc_params* P, const double* G, int32_t ix, int32_t iy,
                        const double* wx, const double* wy, double* out) {
  out[0] = out[1] = out[2] = 0.0;
  for (int b = 0; b < 3; ++b) {
    int32_t yy = iy + b - 1;
    if (yy < 0 || yy >= P->ny) continue;
    for (int a = 0; a < 3; ++a) {
      int32_t xx = ix + a - 1;
      if (xx < 0 || xx >= P->nx) continue;
      const double* m = G + 4 * ((int64_t)yy * P->nx + xx);
      double w = wx[a] * wy[b];
      out[0] += w * m[0];
      out[1] += w * m[1];
      out[2] += w * m[2];
    }
  }
}

/* f at frame-local (u, v) and time weights wt[3] of levels (l0,l1,l2). */
static void integrand(const subctx* X, double u, double v, const double* wt, double* f) {
  const orc_source* S = X->S;
  if (S->kind == ORC_SRC_GRID) {
    const orc_params* P = X->P;
    double tx = u / P->hx, ty = v / P->hy;
    double fx = floor(tx + 0.5), fy = floor(ty + 0.5);
    double wx[3], wy[3];
    if (P->interp == 1) { /* R-25: the time interpolation's quadratic Lagrange in x and y */
      orc_lagrange3_weights(tx - fx, wx);
      orc_lagrange3_weights(ty - fy, wy);
    } else {
      orc_tsc_weights(tx - fx, wx);
      orc_tsc_weights(ty - fy, wy);
    }
    /* clamp far-out indices before the int conversion (values are 0 there) */
    if (fx < -4.0 || fx > P->nx + 4.0 || fy < -4.0 || fy > P->ny + 4.0) {
      f[0] = f[1] = f[2] = 0.0;
      return;
    }
    int32_t ix = (int32_t)fx, iy = (int32_t)fy;
    double g[3][3];
    for (int l = 0; l < 3; ++l) grid_interp(P, X->G[l], ix, iy, wx, wy, g[l]);
    for (int c = 0; c < 3; ++c) f[c] = wt[0] * g[0][c] + wt[1] * g[1][c] + wt[2] * g[2][c];
    return;
  }
  double a = wt[0] * X->amp[0] + wt[1] * X->amp[1] + wt[2] * X->amp[2];
  double rho;
  if (S->kind == ORC_SRC_GAUSS) {
    double ex = u - S->x0, ey = v - S->y0, sg = S->width;
    rho = S->q / (2.0 * M_PI * sg * sg) * exp(-(ex * ex + ey * ey) / (2.0 * sg * sg));
  } else {
    rho = S->q; /* uniform disk, the arc lies inside it */
  }
  rho = a * rho;
  f[0] = rho;
  f[1] = rho * S->bx;
  f[2] = rho * S->by;
}

/* Inner theta integral at radius r ("Newton-Cotes"; R-11): periodic
 * trapezoid on a full circle, composite Simpson with n_theta panels per arc. */
void orc_inner_ctx(subctx* X, double r, double* out) {
  double cu, cv, wt[3];
  centre_at(X, r, &cu, &cv, wt);
  double arcs[16];
  int32_t na;
  if (X->S->kind == ORC_SRC_DISK)
    na = orc_arcs_disk(cu, cv, r, X->S->x0, X->S->y0, X->S->width, arcs);
  else
    na = orc_arcs_rect(cu, cv, r, X->U0, X->U1, X->V0, X->V1, arcs);
  out[0] = out[1] = out[2] = 0.0;
  const int32_t N = X->P->n_theta;
  double f[3];
  if (na < 0) {
    double w = 2.0 * M_PI / N;
    for (int32_t m = 0; m < N; ++m) {
      double th = (double)m * (2.0 * M_PI / N);
      integrand(X, cu + r * cos(th), cv + r * sin(th), wt, f);
      X->evals++;
      for (int c = 0; c < 3; ++c) out[c] += w * f[c];
    }
    return;
  }
  for (int32_t q = 0; q < na; ++q) {
    double t1 = arcs[2 * q], t2 = arcs[2 * q + 1];
    double h = (t2 - t1) / N;
    for (int32_t m = 0; m <= N; ++m) {
      double th = t1 + (double)m * h;
      double w = (m == 0 || m == N) ? h / 3.0 : ((m & 1) ? 4.0 * h / 3.0 : 2.0 * h / 3.0);
      X->evals++;
      /* R-25b: with the Lagrange-3 stencil the integrand jumps on the support boundary, where
       * every arc ends; the end nodes take the limit from outside the support, 0 (under TSC
       * the integrand is continuous there and already 0, R-24) */
      if ((m == 0 || m == N) && X->S->kind == ORC_SRC_GRID && X->P->interp == 1) continue;
      integrand(X, cu + r * cos(th), cv + r * sin(th), wt, f);
      for (int c = 0; c < 3; ++c) out[c] += w * f[c];
    }
  }
}

/* ------------------------------------------------------------------ */
/* GK15 on one segment and the dyadic adaptive tree (*/
/* R-8, R-9, R-10, R-12, R-12b)                                          */
/* ------------------------------------------------------------------ */
static void gk15(subctx* X, double a, double b, double* K, double* G, double* err) {
  double m = 0.5 * (a + b), hw = 0.5 * (b - a);
  double k[3] = {0, 0, 0}, g[3] = {0, 0, 0}, v[3];
  for (int i = 0; i < 7; ++i) {
    orc_inner_ctx(X, m - hw * XGK[i], v);
    for (int c = 0; c < 3; ++c) k[c] += WGK[i] * v[c];
    if (i & 1) for (int c = 0; c < 3; ++c) g[c] += WG[i / 2] * v[c];
    orc_inner_ctx(X, m + hw * XGK[i], v);
    for (int c = 0; c < 3; ++c) k[c] += WGK[i] * v[c];
    if (i & 1) for (int c = 0; c < 3; ++c) g[c] += WG[i / 2] * v[c];
  }
  orc_inner_ctx(X, m, v);
  for (int c = 0; c < 3; ++c) { k[c] += WGK[7] * v[c]; g[c] += WG[3] * v[c]; }
  *err = 0.0;
  for (int c = 0; c < 3; ++c) {
    K[c] = hw * k[c];
    G[c] = hw * g[c];
    double e = fabs(K[c] - G[c]);
    if (e > *err) *err = e;
  }
}

/* The paper's own outer rule (P:155 RP-QUADRULE "standard Simpson's quadrature rule",
 * P:157 Simpson adaptive quadrature; reading R-22): on five equispaced nodes
 * r_0 = a, r_2 = (a+b)/2, r_1 = (r_0+r_2)/2, r_3 = (r_2+r_4)/2, r_4 = b, the composite
 * Simpson estimate S2 = h/12 (1,4,2,4,1) and the single-panel S1 = h/6 (1,0,4,0,1) give the
 * standard error estimate |S2 - S1| / 15 and the Richardson value S2 + (S2 - S1)/15, which
 * is Boole's rule h/90 (7,32,12,32,7).  Returned as K = Boole, G = S2: err = |K - G|. */
static void simpson5(subctx* X, double a, double b, double* K, double* G, double* err) {
  double r[5];
  r[0] = a;
  r[4] = b;
  r[2] = 0.5 * (a + b);
  r[1] = 0.5 * (r[0] + r[2]);
  r[3] = 0.5 * (r[2] + r[4]);
  static const double wb[5] = {7.0, 32.0, 12.0, 32.0, 7.0};
  static const double ws[5] = {1.0, 4.0, 2.0, 4.0, 1.0};
  double h = b - a;
  double kb[3] = {0, 0, 0}, ks[3] = {0, 0, 0}, v[3];
  for (int i = 0; i < 5; ++i) {
    orc_inner_ctx(X, r[i], v);
    for (int c = 0; c < 3; ++c) {
      kb[c] += wb[i] * v[c];
      ks[c] += ws[i] * v[c];
    }
  }
  *err = 0.0;
  for (int c = 0; c < 3; ++c) {
    K[c] = h / 90.0 * kb[c];
    G[c] = h / 12.0 * ks[c];
    double e = fabs(K[c] - G[c]);
    if (e > *err) *err = e;
  }
}

/* depth-first, left to right: visit (level, index) on [A,B] */
static void tree(subctx* X, double A, double B, double R, int32_t lev, int64_t idx,
                 orc_result* res) {
  const orc_params* P = X->P;
  double fa = ldexp((double)idx, -lev), fb = ldexp((double)(idx + 1), -lev);
  double a = A + (B - A) * fa, b = A + (B - A) * fb;
  double K[3], G[3], err;
  const int64_t e0 = X->evals;
  if (P->rule == 1)
    simpson5(X, a, b, K, G, &err);
  else
    gk15(X, a, b, K, G, &err);
  const int64_t de = X->evals - e0;
  res->nseg++;
  res->nodes += P->rule == 1 ? 5 : 15;
  double tol = P->tau * ldexp(B - A, -lev) / R;
  double margin = fabs(err - tol) / tol;
  if (margin < res->min_margin) res->min_margin = margin;
  if (margin < 1e-9) res->ties++;
  /* R-28: err = max_c |K_c - G_c| is a difference of two nearly equal sums; a different
   * (equally valid) summation order moves it by a few ulp of |K| + |G| (rho component: it
   * bounds the current components, |J| <= rho), so a decision whose margin lies within that
   * noise is decided by rounding, not by R-10.  Diagnostic only: the tree is unchanged. */
  const double scale = DBL_EPSILON * (fabs(K[0]) + fabs(G[0]));
  const double noise = scale > 0.0 ? fabs(err - tol) / scale : INFINITY;
  if (noise < res->min_noise) res->min_noise = noise;
  if (noise < ORC_NOISE_TIE) res->noise_ties++;
  if (lev > res->max_level) res->max_level = lev;
  if (err <= tol || lev >= P->max_depth) {
    if (!(err <= tol)) {
      res->capped++;
      res->chase_segs++;
      res->chase_evals += de;
    }
    res->nleaf++;
    if (X->ends) { X->ends[X->nends++] = a; X->last_b = b; }  /* DFS order = ascending r' */
    res->phi += K[0];
    res->ax += K[1];
    res->ay += K[2];
    res->err += err;
    return;
  }
  const int32_t capped0 = res->capped;
  tree(X, A, B, R, lev + 1, 2 * idx, res);
  tree(X, A, B, R, lev + 1, 2 * idx + 1, res);
  if (res->capped > capped0) {  /* this segment split on the way to a capped leaf */
    res->chase_segs++;
    res->chase_evals += de;
  }
}

/* ------------------------------------------------------------------ */
/* rp-integral at one mesh point (Eq. 1-2; C.3)                 */
/* ------------------------------------------------------------------ */
int32_t orc_kappa(const orc_params* P, const orc_hist* Hh) {
  int32_t kap = Hh->k + Hh->n_pre - 1;
  if (kap > P->kappa_max) kap = P->kappa_max;
  if (kap < 0) kap = 0;
  return kap;
}

static void setup_sub(subctx* X, const orc_params* P, const orc_hist* Hh, const orc_source* S,
                      double px, double py, int32_t j) {
  memset(X, 0, sizeof(*X));
  X->P = P; X->Hh = Hh; X->S = S; X->px = px; X->py = py; X->j = j;
  for (int l = 0; l < 3; ++l) {
    int32_t level = Hh->k - j - 2 + l;
    int32_t sl = slot_of(level, Hh->H);
    X->F[l] = Hh->frames + sl;
    X->G[l] = Hh->ring ? Hh->ring + (int64_t)sl * P->ny * P->nx * 4 : NULL;
    X->amp[l] = S->amp ? S->amp[sl] : 1.0;
  }
  if (S->kind == ORC_SRC_GAUSS) {
    X->U0 = S->x0 - 8.0 * S->width; X->U1 = S->x0 + 8.0 * S->width;
    X->V0 = S->y0 - 8.0 * S->width; X->V1 = S->y0 + 8.0 * S->width;
  } else {
    X->U0 = -1.5 * P->hx; X->U1 = (P->nx + 0.5) * P->hx;
    X->V0 = -1.5 * P->hy; X->V1 = (P->ny + 0.5) * P->hy;
  }
}

/* Mesh node (ix,iy) of the frame of step k, in the lab. */
void orc_mesh_point(const orc_params* P, const orc_frame* F, int32_t ix, int32_t iy,
                    double* px, double* py) {
  double u = ix * P->hx, v = iy * P->hy;
  *px = F->ox + u * F->c - v * F->s;
  *py = F->oy + u * F->s + v * F->c;
}

/* Root intervals of one (point, subregion) item under the Predictive-RP variant (R-26):
 * the intervals of the item's cluster partition list (sorted breakpoints of S_j) cut to
 * the item's support [A, B]; empty pieces dropped. */
typedef struct {
  const double* bp;      /* breakpoints, all lists back to back                         */
  const int64_t* off;    /* [n_clusters * kappa_max + 1]: list (c, j) = bp[off[i], off[i+1]) */
  int32_t cluster;       /* the point's cluster                                          */
  int32_t kappa_max;
} orc_roots;

/* parts (nullable): the item partitions -- for each j with accepted leaves, the leaves' left
 * ends in r' order followed by the last leaf's right end, written at parts + parts_off[j]
 * (parts_off [kappa_max], from a first call's leaf counts: count + 1 doubles per item). */
static void point_lab_ex(const orc_params* P, const orc_hist* Hh, const orc_source* S,
                         double px, double py, const orc_roots* RT, uint16_t* leaves_row,
                         const int64_t* parts_off, double* parts, orc_result* res) {
  memset(res, 0, sizeof(*res));
  res->min_margin = INFINITY;
  res->min_noise = INFINITY;
  int32_t kap = orc_kappa(P, Hh);
  if (kap == 0) return;
  double cdt = P->c * P->dt;
  double R = kap * cdt;
  for (int32_t j = 0; j < kap; ++j) {
    subctx X;
    setup_sub(&X, P, Hh, S, px, py, j);
    double A, B;
    if (!orc_clip(&X, j * cdt, (j + 1) * cdt, &A, &B)) continue;
    int32_t leaves0 = res->nleaf;
    if (parts) X.ends = parts + parts_off[j];
    int64_t lo = 0, hi = 0;
    if (RT) {
      int64_t i = (int64_t)RT->cluster * RT->kappa_max + j;
      lo = RT->off[i];
      hi = RT->off[i + 1];
    }
    if (hi - lo >= 2) {
      /* Algorithm 1 lines 13-16 (COMPUTE-RP-INTEGRAL over the cluster partition) and 18-24
       * (adaptive quadrature on the intervals that fail): each cut interval is the root of
       * a dyadic tree, its first evaluation being the partition-phase estimate */
      for (int64_t t = lo; t + 1 < hi; ++t) {
        double a = RT->bp[t] > A ? RT->bp[t] : A;
        double b = RT->bp[t + 1] < B ? RT->bp[t + 1] : B;
        if (a < b) tree(&X, a, b, R, 0, 0, res);
      }
    } else if (P->n_root == 1) {
      tree(&X, A, B, R, 0, 0, res);
    } else if (P->n_root == 4 && j > 0) {  /* variant: the four quarters of [A, B] */
      for (int64_t q = 0; q < 4; ++q) tree(&X, A, B, R, 2, q, res);
    } else if (j == 0) {
      /* R-12b: the near field S_0 (r' from 0) starts from the 2^L equal pieces of [A, B] no
       * longer than an eighth of the grid's extent L_g = max(nx hx, ny hy) -- the scale of the
       * comoving bunch's structure that the first r' of the light cone sweep -- with
       * 2 <= L <= 7: the smallest such L, by exact power-of-two comparisons */
      const double Lg = P->nx * P->hx > P->ny * P->hy ? P->nx * P->hx : P->ny * P->hy;
      int32_t L = 2;
      while (L < 7 && B - A > ldexp(Lg, L - 3)) ++L;
      for (int64_t q = 0; q < ((int64_t)1 << L); ++q) tree(&X, A, B, R, L, q, res);
    } else {
      tree(&X, A, B, R, 1, 0, res);
      tree(&X, A, B, R, 1, 1, res);
    }
    /* the leaves tile [A, B]; the list closes with the last leaf's right end as the tree
     * computed it (A + (B - A) * 1, which may differ from B in the last bit) */
    if (X.ends && X.nends > 0) X.ends[X.nends++] = X.last_b;
    if (leaves_row) {
      int32_t nl = res->nleaf - leaves0;
      leaves_row[j] = (uint16_t)(nl < 0xFFFF ? nl : 0xFFFF);
    }
    res->evals += X.evals;
  }
}

void orc_point_lab(const orc_params* P, const orc_hist* Hh, const orc_source* S, double px,
                   double py, orc_result* res) {
  point_lab_ex(P, Hh, S, px, py, NULL, NULL, NULL, NULL, res);
}

/* Potentials at a list of mesh points (flattened iy*nx+ix) of frame k.  leaves (nullable):
 * [npts][kappa_max] accepted segments per (point, subregion) -- the observed access
 * pattern n_j(p) of P:83-95 that the Predictive-RP variant forecasts from. */
void orc_potentials_ex(const orc_params* P, const orc_hist* Hh, const orc_source* S,
                       const int32_t* pts, int32_t npts, uint16_t* leaves, orc_result* out) {
  const orc_frame* Fk = Hh->frames + slot_of(Hh->k, Hh->H);
#pragma omp parallel for schedule(dynamic, 1)
  for (int32_t i = 0; i < npts; ++i) {
    int32_t p = pts[i];
    double px, py;
    orc_mesh_point(P, Fk, p % P->nx, p / P->nx, &px, &py);
    uint16_t* row = leaves ? leaves + (int64_t)i * P->kappa_max : NULL;
    if (row) memset(row, 0, sizeof(uint16_t) * P->kappa_max);
    point_lab_ex(P, Hh, S, px, py, NULL, row, NULL, NULL, out + i);
  }
}

/* The accepted partitions of every item (P:104's "partition generated at an earlier time
 * step"): off [npts * kappa_max], point i's item j written at parts + off[i * kappa_max + j]
 * (leaf left ends in r' order, then the last right end; nothing for an item without leaves).
 * The offsets come from the leaf counts of orc_potentials_ex on the same state. */
void orc_potentials_parts(const orc_params* P, const orc_hist* Hh, const orc_source* S,
                          const int32_t* pts, int32_t npts, const int64_t* off, double* parts,
                          orc_result* out) {
  const orc_frame* Fk = Hh->frames + slot_of(Hh->k, Hh->H);
#pragma omp parallel for schedule(dynamic, 1)
  for (int32_t i = 0; i < npts; ++i) {
    int32_t p = pts[i];
    double px, py;
    orc_mesh_point(P, Fk, p % P->nx, p / P->nx, &px, &py);
    point_lab_ex(P, Hh, S, px, py, NULL, NULL, off + (int64_t)i * P->kappa_max, parts, out + i);
  }
}

void orc_potentials(const orc_params* P, const orc_hist* Hh, const orc_source* S,
                    const int32_t* pts, int32_t npts, orc_result* out) {
  orc_potentials_ex(P, Hh, S, pts, npts, NULL, out);
}

/* ------------------------------------------------------------------ */
/* Predictive-RP: the paper's COMPUTE-POTENTIALS (Algorithm 1) as a variant    */
/* (reading R-26).  Lines 1-6 and 9-12 are host work in the paper; here they are   */
/* written out plainly, in the paper's order.                                              */
/* ------------------------------------------------------------------ */
/* Line 3, g = kNN regression over the mesh: the mean of the previous step's access
 * pattern n_j over the k nearest mesh nodes in index space (k = 1: the node; 5: the node and
 * its 4 edge neighbours; 9: the 3x3 block; 25: the 5x5 block; nodes off the mesh are not
 * neighbours), rounded half up: (sum + cnt/2) / cnt in integers. */
int32_t orc_knn_pattern(const uint16_t* prev, int32_t nx, int32_t ny, int32_t kmax, int32_t p,
                        int32_t j, int32_t knn) {
  int32_t ix = p % nx, iy = p / nx;
  int32_t rad = knn >= 25 ? 2 : (knn >= 5 ? 1 : 0);
  uint32_t sum = 0, cnt = 0;
  for (int32_t dy = -rad; dy <= rad; ++dy)
    for (int32_t dx = -rad; dx <= rad; ++dx) {
      if (knn == 5 && dx != 0 && dy != 0) continue;
      int32_t x = ix + dx, y = iy + dy;
      if (x < 0 || x >= nx || y < 0 || y >= ny) continue;
      sum += prev[((int64_t)y * nx + x) * kmax + j];
      cnt++;
    }
  return (int32_t)((sum + cnt / 2) / cnt);
}

/* Line 6, RP-CLUSTERING: k-means of the access-pattern vectors
 * a(p) = (n_0(p) .. n_{kmax-1}(p)) into m clusters.  Deterministic reading (R-26): initial
 * centres a(p_c) with p_c = floor(c * npts / m); Lloyd iterations -- assign every point to
 * the centre of least squared distance (sum over j ascending of (a_j - mu_j)^2, ties to the
 * lower c), then every non-empty cluster's centre to the mean of its members (integer sums
 * divided once) -- until no assignment changes or max_iters assignments were made.
 * Returns the number of assignment passes. */
int32_t orc_kmeans(const uint16_t* pat, int32_t npts, int32_t kmax, int32_t m, int32_t max_iters,
                   int32_t* assign) {
  double* mu = (double*)malloc(sizeof(double) * (size_t)m * kmax);
  int64_t* sum = (int64_t*)malloc(sizeof(int64_t) * (size_t)m * kmax);
  int64_t* cnt = (int64_t*)malloc(sizeof(int64_t) * (size_t)m);
  for (int32_t c = 0; c < m; ++c) {
    int64_t pc = (int64_t)c * npts / m;
    for (int32_t j = 0; j < kmax; ++j) mu[(int64_t)c * kmax + j] = (double)pat[pc * kmax + j];
  }
  for (int32_t p = 0; p < npts; ++p) assign[p] = -1;
  int32_t it = 0;
  for (;;) {
    int32_t changed = 0;
    ++it;
    for (int32_t p = 0; p < npts; ++p) {
      int32_t best = 0;
      double bd = INFINITY;
      for (int32_t c = 0; c < m; ++c) {
        double d = 0.0;
        for (int32_t j = 0; j < kmax; ++j) {
          double e = (double)pat[(int64_t)p * kmax + j] - mu[(int64_t)c * kmax + j];
          d += e * e;
        }
        if (d < bd) { bd = d; best = c; }
      }
      if (assign[p] != best) { assign[p] = best; changed = 1; }
    }
    if (!changed || it >= max_iters) break;
    memset(sum, 0, sizeof(int64_t) * (size_t)m * kmax);
    memset(cnt, 0, sizeof(int64_t) * (size_t)m);
    for (int32_t p = 0; p < npts; ++p) {
      cnt[assign[p]]++;
      for (int32_t j = 0; j < kmax; ++j) sum[(int64_t)assign[p] * kmax + j] += pat[(int64_t)p * kmax + j];
    }
    for (int32_t c = 0; c < m; ++c)
      if (cnt[c] > 0)
        for (int32_t j = 0; j < kmax; ++j)
          mu[(int64_t)c * kmax + j] = (double)sum[(int64_t)c * kmax + j] / (double)cnt[c];
  }
  free(mu); free(sum); free(cnt);
  return it;
}


/* Lines 4 and 9-12: COMPUTE-PARTITION by uniform partitioning (n_j(p) equal pieces of
 * S_j = [j c dt, (j+1) c dt], breakpoints a_j + (b_j - a_j) * (t / n), the last one b_j
 * itself so the list covers S_j exactly), then MERGE-LISTS over
 * the members of each cluster (sorted, duplicate values removed).  off has
 * m * kmax + 1 entries; bp (nullable: count only) receives the lists.  A point with
 * n_j(p) = 0 contributes nothing; an empty list means "no forecast" (canonical roots). */
/* Line 4 by adaptive partitioning (reading R-26b): a member p whose item (p, j) had an
 * accepted partition x_0 < ... < x_d at the earlier step (prev_parts + prev_off[p * kmax + j],
 * prev_len[...] = d + 1 doubles) divides each of its d pieces into q = max(1, round(n/d))
 * equal pieces, n = n_j(p) the forecast (q = (2n + d) / (2d) in integers: half up), with
 * breakpoints x_{i-1} + (x_i - x_{i-1}) * (t / q), the last one x_i itself; a_j and b_j are
 * added so the list covers S_j (pieces outside the earlier support stay whole).  A member
 * without an earlier partition of S_j uses uniform partitioning.  MERGE-LISTS as above. */
static int64_t adaptive_list(const orc_params* P, const uint16_t* pat, const int32_t* assign,
                             int32_t npts, int32_t c, int32_t j, const int64_t* prev_off,
                             const int32_t* prev_len, const double* prev_parts, double** buf,
                             int64_t* cap) {
  const int32_t kmax = P->kappa_max;
  const double cdt = P->c * P->dt;
  const double aj = j * cdt, bj = (j + 1) * cdt;
  int64_t need = 0;
  for (int32_t p = 0; p < npts; ++p) {
    int32_t n = pat[(int64_t)p * kmax + j];
    if (assign[p] != c || n == 0) continue;
    int32_t len = prev_len[(int64_t)p * kmax + j];
    if (len >= 2) {
      int32_t d = len - 1, q = (2 * n + d) / (2 * d);
      if (q < 1) q = 1;
      need += (int64_t)d * q + 1 + 2;
    } else {
      need += n + 1;
    }
  }
  if (need > *cap) {
    *cap = need;
    *buf = (double*)realloc(*buf, sizeof(double) * (size_t)need);
  }
  double* L = *buf;
  int64_t u = 0;
  for (int32_t p = 0; p < npts; ++p) {
    int32_t n = pat[(int64_t)p * kmax + j];
    if (assign[p] != c || n == 0) continue;
    int32_t len = prev_len[(int64_t)p * kmax + j];
    if (len >= 2) {
      const double* x = prev_parts + prev_off[(int64_t)p * kmax + j];
      int32_t d = len - 1, q = (2 * n + d) / (2 * d);
      if (q < 1) q = 1;
      L[u++] = aj;
      L[u++] = bj;
      for (int32_t i = 1; i <= d; ++i)
        for (int32_t t = 0; t < q; ++t) L[u++] = x[i - 1] + (x[i] - x[i - 1]) * ((double)t / (double)q);
      L[u++] = x[d];
    } else {
      for (int32_t t = 0; t <= n; ++t) L[u++] = t == n ? bj : aj + (bj - aj) * ((double)t / (double)n);
    }
  }
  return u;
}

int64_t orc_merge_partitions_mode(const orc_params* P, const uint16_t* pat, const int32_t* assign,
                                  int32_t npts, int32_t m, int32_t mode, const int64_t* prev_off,
                                  const int32_t* prev_len, const double* prev_parts, int64_t* off,
                                  double* bp);

int64_t orc_merge_partitions(const orc_params* P, const uint16_t* pat, const int32_t* assign,
                             int32_t npts, int32_t m, int64_t* off, double* bp) {
  return orc_merge_partitions_mode(P, pat, assign, npts, m, 0, NULL, NULL, NULL, off, bp);
}

/* mode 0: uniform partitioning; 1: adaptive partitioning (needs the earlier
 * partitions prev_off / prev_len / prev_parts of all npts points). */
int64_t orc_merge_partitions_mode(const orc_params* P, const uint16_t* pat, const int32_t* assign,
                                  int32_t npts, int32_t m, int32_t mode, const int64_t* prev_off,
                                  const int32_t* prev_len, const double* prev_parts, int64_t* off,
                                  double* bp) {
  const int32_t kmax = P->kappa_max;
  const double cdt = P->c * P->dt;
  int64_t total = 0;
  uint8_t* seen = (uint8_t*)calloc(65536, 1);
  double* buf = NULL;
  int64_t cap = 0;
  for (int32_t c = 0; c < m; ++c)
    for (int32_t j = 0; j < kmax; ++j) {
      off[(int64_t)c * kmax + j] = total;
      if (mode == 1) {
        int64_t q = adaptive_list(P, pat, assign, npts, c, j, prev_off, prev_len, prev_parts,
                                  &buf, &cap);
        if (q) qsort(buf, (size_t)q, sizeof(double), cmp_double);
        int64_t u = 0;
        for (int64_t i = 0; i < q; ++i)
          if (u == 0 || buf[i] != buf[u - 1]) buf[u++] = buf[i];
        if (bp) memcpy(bp + total, buf, sizeof(double) * (size_t)u);
        total += u;
        continue;
      }
      memset(seen, 0, 65536);
      int64_t n_all = 0;
      for (int32_t p = 0; p < npts; ++p) {
        int32_t n = pat[(int64_t)p * kmax + j];
        if (assign[p] != c || n == 0 || seen[n]) continue;
        seen[n] = 1;
        n_all += n + 1;
      }
      if (n_all > cap) {
        cap = n_all;
        buf = (double*)realloc(buf, sizeof(double) * (size_t)cap);
      }
      double a = j * cdt, b = (j + 1) * cdt;
      int64_t q = 0;
      for (int32_t n = 1; n < 65536; ++n) {
        if (!seen[n]) continue;
        for (int32_t t = 0; t <= n; ++t) buf[q++] = t == n ? b : a + (b - a) * ((double)t / (double)n);
      }
      if (q) qsort(buf, (size_t)q, sizeof(double), cmp_double);
      int64_t u = 0;
      for (int64_t i = 0; i < q; ++i)
        if (u == 0 || buf[i] != buf[u - 1]) buf[u++] = buf[i];
      if (bp) memcpy(bp + total, buf, sizeof(double) * (size_t)u);
      total += u;
    }
  off[(int64_t)m * kmax] = total;
  free(seen);
  free(buf);
  return total;
}

/* The whole variant for step k (Algorithm 1 lines 1-24): prev = the previous step's observed
 * pattern [nx*ny][kmax] (e.g. from orc_potentials_ex); m = number of clusters (0: max(nx,
 * ny)).  Writes the clusters (nullable) and the results at pts; leaves (nullable) as
 * in orc_potentials_ex.  Returns the number of k-means assignment passes. */
int32_t orc_potentials_predictive2(const orc_params* P, const orc_hist* Hh, const orc_source* S,
                                   const uint16_t* prev, int32_t knn, int32_t m,
                                   int32_t max_iters, int32_t mode, const int64_t* prev_off,
                                   const int32_t* prev_len, const double* prev_parts,
                                   const int32_t* pts, int32_t npts, int32_t* cluster_out,
                                   uint16_t* leaves, orc_result* out);

int32_t orc_potentials_predictive(const orc_params* P, const orc_hist* Hh, const orc_source* S,
                                  const uint16_t* prev, int32_t knn, int32_t m,
                                  int32_t max_iters, const int32_t* pts, int32_t npts,
                                  int32_t* cluster_out, uint16_t* leaves, orc_result* out) {
  return orc_potentials_predictive2(P, Hh, S, prev, knn, m, max_iters, 0, NULL, NULL, NULL, pts,
                                    npts, cluster_out, leaves, out);
}

/* mode 0: uniform partitioning; mode 1: adaptive partitioning from the earlier
 * step's accepted partitions of all nx*ny points (prev_off / prev_len [nx*ny * kmax], as
 * written by orc_potentials_parts). */
int32_t orc_potentials_predictive2(const orc_params* P, const orc_hist* Hh, const orc_source* S,
                                   const uint16_t* prev, int32_t knn, int32_t m,
                                   int32_t max_iters, int32_t mode, const int64_t* prev_off,
                                   const int32_t* prev_len, const double* prev_parts,
                                   const int32_t* pts, int32_t npts, int32_t* cluster_out,
                                   uint16_t* leaves, orc_result* out) {
  const int32_t nx = P->nx, ny = P->ny, kmax = P->kappa_max, nall = nx * ny;
  const int32_t kap = orc_kappa(P, Hh);
  if (m <= 0) m = nx > ny ? nx : ny;
  if (m > nall) m = nall;
  uint16_t* pat = (uint16_t*)calloc((size_t)nall * kmax, sizeof(uint16_t));
  for (int32_t p = 0; p < nall; ++p)
    for (int32_t j = 0; j < kap; ++j)
      pat[(int64_t)p * kmax + j] = (uint16_t)orc_knn_pattern(prev, nx, ny, kmax, p, j, knn);
  int32_t* assign = (int32_t*)malloc(sizeof(int32_t) * nall);
  int32_t iters = orc_kmeans(pat, nall, kmax, m, max_iters, assign);
  int64_t* off = (int64_t*)malloc(sizeof(int64_t) * ((size_t)m * kmax + 1));
  int64_t nbp = orc_merge_partitions_mode(P, pat, assign, nall, m, mode, prev_off, prev_len,
                                          prev_parts, off, NULL);
  double* bp = (double*)malloc(sizeof(double) * (size_t)(nbp > 0 ? nbp : 1));
  orc_merge_partitions_mode(P, pat, assign, nall, m, mode, prev_off, prev_len, prev_parts, off,
                            bp);
  const orc_frame* Fk = Hh->frames + slot_of(Hh->k, Hh->H);
#pragma omp parallel for schedule(dynamic, 1)
  for (int32_t i = 0; i < npts; ++i) {
    int32_t p = pts[i];
    double px, py;
    orc_mesh_point(P, Fk, p % nx, p / nx, &px, &py);
    orc_roots RT = {bp, off, assign[p], kmax};
    uint16_t* row = leaves ? leaves + (int64_t)i * kmax : NULL;
    if (row) memset(row, 0, sizeof(uint16_t) * kmax);
    point_lab_ex(P, Hh, S, px, py, &RT, row, NULL, NULL, out + i);
  }
  if (cluster_out) memcpy(cluster_out, assign, sizeof(int32_t) * nall);
  free(pat); free(assign); free(off); free(bp);
  return iters;
}

/* Test hooks: the clip, inner integral and a single tree for (point, j). */
int32_t orc_clip_at(const orc_params* P, const orc_hist* Hh, const orc_source* S, double px,
                    double py, int32_t j, double* A, double* B) {
  subctx X;
  setup_sub(&X, P, Hh, S, px, py, j);
  double cdt = P->c * P->dt;
  return orc_clip(&X, j * cdt, (j + 1) * cdt, A, B);
}

void orc_dists_at(const orc_params* P, const orc_hist* Hh, const orc_source* S, double px,
                  double py, int32_t j, double r, double* dmin2, double* dmax2) {
  subctx X;
  setup_sub(&X, P, Hh, S, px, py, j);
  dists_at(&X, r, dmin2, dmax2);
}

/* Frame-local centre (c_u, c_v) of the circle about lab point p at radius r of subregion j,
 * i.e. p in the frame interpolated to the retarded time t' = k dt - r/c (R-7), and the time
 * weights of levels (l0, l1, l2) there. */
void orc_centre_at(const orc_params* P, const orc_hist* Hh, const orc_source* S, double px,
                   double py, int32_t j, double r, double* cu, double* cv, double* w) {
  subctx X;
  setup_sub(&X, P, Hh, S, px, py, j);
  centre_at(&X, r, cu, cv, w);
}

int64_t orc_inner_at(const orc_params* P, const orc_hist* Hh, const orc_source* S, double px,
                     double py, int32_t j, double r, double* out) {
  subctx X;
  setup_sub(&X, P, Hh, S, px, py, j);
  orc_inner_ctx(&X, r, out);
  return X.evals;
}

void orc_integrand_at(const orc_params* P, const orc_hist* Hh, const orc_source* S,
                      int32_t j, double u, double v, double tau_t, double* f) {
  subctx X;
  setup_sub(&X, P, Hh, S, 0.0, 0.0, j);
  double wt[3];
  orc_lagrange3_weights(tau_t, wt);
  integrand(&X, u, v, wt, f);
}

void orc_gk15_at(const orc_params* P, const orc_hist* Hh, const orc_source* S, double px,
                 double py, int32_t j, double a, double b, double* K, double* G, double* err) {
  subctx X;
  setup_sub(&X, P, Hh, S, px, py, j);
  gk15(&X, a, b, K, G, err);
}

/* ------------------------------------------------------------------ */
/* Self-fields (R-15)                                  */
/* ------------------------------------------------------------------ */
static double d_dir(const double* f, int32_t nx, int32_t ny, int32_t ix, int32_t iy, int dir,
                    double h) {
  int32_t n = dir == 0 ? nx : ny, i = dir == 0 ? ix : iy;
#define AT(o) (dir == 0 ? f[(int64_t)iy * nx + (ix + (o))] : f[(int64_t)(iy + (o)) * nx + ix])
  if (i == 0) return (-3.0 * AT(0) + 4.0 * AT(1) - AT(2)) / (2.0 * h);
  if (i == n - 1) return (3.0 * AT(0) - 4.0 * AT(-1) + AT(-2)) / (2.0 * h);
  return (AT(1) - AT(-1)) / (2.0 * h);
#undef AT
}

/* Backward-difference weights of order m = 1..4 for f'(t_k) from f(t_k), ..., f(t_{k-m}),
 * in units of 1/dt (exact for polynomials of degree m; R-15b). */
static const double BD[5][5] = {{0, 0, 0, 0, 0},
                                {1.0, -1.0, 0, 0, 0},
                                {1.5, -2.0, 0.5, 0, 0},
                                {11.0 / 6.0, -3.0, 1.5, -1.0 / 3.0, 0},
                                {25.0 / 12.0, -4.0, 3.0, -4.0 / 3.0, 0.25}};

/* E = -grad(phi) - (1/c) dA/dt ,  B_z = d_x A_y - d_y A_x  on mesh k (R-15b).
 * The mesh moves with its frame, so the lab time derivative at a node is the derivative
 * following the node minus the convective term:
 *   dA/dt|lab = (1/dt) sum_j BD[m][j] A_{k-j}(node)  -  (V . grad) A_k,
 *   V = (1/dt) sum_j BD[m][j] P_{k-j}(node),
 * both order-m backward differences at t_k (j = 0..m) on the same nodes, so a field at rest in
 * the lab cancels exactly and one co-moving with the mesh is exact to O(dt^m).
 * fr[0..m]: frames of levels k, k-1, ..., k-m; a_prev [m][2][ny*nx]: (A_x, A_y) of steps
 * k-1, ..., k-m (most recent first); m = 0 omits the dA/dt term. */
void orc_fields(const orc_params* P, const orc_frame* fr, int32_t m, const double* phi,
                const double* ax, const double* ay, const double* a_prev, double* ex, double* ey,
                double* bz) {
  const int32_t nx = P->nx, ny = P->ny;
  const int64_t npts = (int64_t)nx * ny;
  const orc_frame* Fk = fr;
  for (int32_t iy = 0; iy < ny; ++iy)
    for (int32_t ix = 0; ix < nx; ++ix) {
      int64_t id = (int64_t)iy * nx + ix;
      double c = Fk->c, s = Fk->s;
      double pu = d_dir(phi, nx, ny, ix, iy, 0, P->hx), pv = d_dir(phi, nx, ny, ix, iy, 1, P->hy);
      double xu = d_dir(ax, nx, ny, ix, iy, 0, P->hx), xv = d_dir(ax, nx, ny, ix, iy, 1, P->hy);
      double yu = d_dir(ay, nx, ny, ix, iy, 0, P->hx), yv = d_dir(ay, nx, ny, ix, iy, 1, P->hy);
      double phx = c * pu - s * pv, phy = s * pu + c * pv;
      double axx = c * xu - s * xv, axy = s * xu + c * xv; /* d_x A_x, d_y A_x */
      double ayx = c * yu - s * yv, ayy = s * yu + c * yv; /* d_x A_y, d_y A_y */
      double dax = 0.0, day = 0.0;
      if (a_prev && m >= 1) {
        double vx = 0.0, vy = 0.0, nax = BD[m][0] * ax[id], nay = BD[m][0] * ay[id];
        for (int32_t j = 0; j <= m; ++j) {
          double px, py;
          orc_mesh_point(P, fr + j, ix, iy, &px, &py);
          vx += BD[m][j] * px;
          vy += BD[m][j] * py;
          if (j >= 1) {
            nax += BD[m][j] * a_prev[(int64_t)(j - 1) * 2 * npts + id];
            nay += BD[m][j] * a_prev[(int64_t)(j - 1) * 2 * npts + npts + id];
          }
        }
        dax = (nax - (vx * axx + vy * axy)) / P->dt;
        day = (nay - (vx * ayx + vy * ayy)) / P->dt;
      }
      ex[id] = -phx - dax / P->c;
      ey[id] = -phy - day / P->c;
      bz[id] = ayx - axy;
    }
}

/* ------------------------------------------------------------------ */
/* Push (P:60 leap-frog Lorentz; R-15): relativistic Boris   */
/* ------------------------------------------------------------------ */
static double gather_tsc(const orc_params* P, const double* F, int32_t ix, int32_t iy,
                         const double* wx, const double* wy) {
  double s = 0.0;
  for (int b = 0; b < 3; ++b) {
    int32_t yy = iy + b - 1;
    if (yy < 0 || yy >= P->ny) continue;
    for (int a = 0; a < 3; ++a) {
      int32_t xx = ix + a - 1;
      if (xx < 0 || xx >= P->nx) continue;
      s += wx[a] * wy[b] * F[(int64_t)yy * P->nx + xx];
    }
  }
  return s;
}

void orc_push(const orc_params* P, const orc_frame* Fk, int64_t n, double* x, double* y,
              double* ux, double* uy, double q_over_mc, double bz_ext, const double* ex,
              const double* ey, const double* bz) {
  for (int64_t i = 0; i < n; ++i) {
    double u, v;
    to_local(Fk, x[i], y[i], &u, &v);
    double tx = u / P->hx, ty = v / P->hy;
    double fx = floor(tx + 0.5), fy = floor(ty + 0.5);
    double Ex = 0.0, Ey = 0.0, Bz = 0.0;
    if (fx >= -2.0 && fx <= P->nx + 1.0 && fy >= -2.0 && fy <= P->ny + 1.0) {
      double wx[3], wy[3];
      orc_tsc_weights(tx - fx, wx);
      orc_tsc_weights(ty - fy, wy);
      int32_t ix = (int32_t)fx, iy = (int32_t)fy;
      Ex = gather_tsc(P, ex, ix, iy, wx, wy);
      Ey = gather_tsc(P, ey, ix, iy, wx, wy);
      Bz = gather_tsc(P, bz, ix, iy, wx, wy);
    }
    Bz += bz_ext;
    double h = 0.5 * q_over_mc * P->dt;
    double umx = ux[i] + h * Ex, umy = uy[i] + h * Ey;
    double gm = sqrt(1.0 + umx * umx + umy * umy);
    double t = h * Bz / gm;
    double sr = 2.0 * t / (1.0 + t * t);
    double upx = umx + umy * t, upy = umy - umx * t;
    double ppx = umx + upy * sr, ppy = umy - upx * sr;
    double nux = ppx + h * Ex, nuy = ppy + h * Ey;
    double g = sqrt(1.0 + nux * nux + nuy * nuy);
    ux[i] = nux;
    uy[i] = nuy;
    x[i] += P->c * P->dt * nux / g;
    y[i] += P->c * P->dt * nuy / g;
  }
}

/* Time-centred momenta for the current (R-27): the leap-frog momenta live at t_k - dt/2 (P:60,
 * R-21), the current of step k at t_k, so the loop deposits u advanced by frac * dt in the
 * uniform external B_z -- the Boris rotation of orc_push with E = 0 and step frac * dt (the
 * self-field part of that half step is below 1e-6 relative in the bend and the previous step's
 * fields live on the previous mesh, which the bunch has left; it is not included). */
void orc_kick_external(const orc_params* P, int64_t n, const double* ux, const double* uy,
                       double q_over_mc, double bz_ext, double frac, double* ux_out,
                       double* uy_out) {
  for (int64_t i = 0; i < n; ++i) {
    double h = 0.5 * q_over_mc * (frac * P->dt);
    double gm = sqrt(1.0 + ux[i] * ux[i] + uy[i] * uy[i]);
    double t = h * bz_ext / gm;
    double sr = 2.0 * t / (1.0 + t * t);
    double upx = ux[i] + uy[i] * t, upy = uy[i] - ux[i] * t;
    ux_out[i] = ux[i] + upy * sr;
    uy_out[i] = uy[i] - upx * sr;
  }
}

/* Lorentz force per unit charge on each particle (the particle-level force F_i of the paper's
 * validation): F = E + beta x (B_z + B_ext) z-hat with (E, B_z) gathered at the
 * particle by the push's TSC weights (R-15) and beta = u / gamma.
 *   F_x = E_x + beta_y B_z,   F_y = E_y - beta_x B_z. */
void orc_forces(const orc_params* P, const orc_frame* Fk, int64_t n, const double* x,
                const double* y, const double* ux, const double* uy, double bz_ext,
                const double* ex, const double* ey, const double* bz, double* fx, double* fy) {
  for (int64_t i = 0; i < n; ++i) {
    double u, v;
    to_local(Fk, x[i], y[i], &u, &v);
    double tx = u / P->hx, ty = v / P->hy;
    double gx = floor(tx + 0.5), gy = floor(ty + 0.5);
    double Ex = 0.0, Ey = 0.0, Bz = 0.0;
    if (gx >= -2.0 && gx <= P->nx + 1.0 && gy >= -2.0 && gy <= P->ny + 1.0) {
      double wx[3], wy[3];
      orc_tsc_weights(tx - gx, wx);
      orc_tsc_weights(ty - gy, wy);
      int32_t ix = (int32_t)gx, iy = (int32_t)gy;
      Ex = gather_tsc(P, ex, ix, iy, wx, wy);
      Ey = gather_tsc(P, ey, ix, iy, wx, wy);
      Bz = gather_tsc(P, bz, ix, iy, wx, wy);
    }
    Bz += bz_ext;
    double g = sqrt(1.0 + ux[i] * ux[i] + uy[i] * uy[i]);
    fx[i] = Ex + (uy[i] / g) * Bz;
    fy[i] = Ey - (ux[i] / g) * Bz;
  }
}
