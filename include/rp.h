/*
 * rp.h -- C ABI of librp, the B200-native retarded-potential step of
 *   Arumugam et al., "A Machine Learning Approach for Efficient Parallel
 *   Simulation of Beam Dynamics on GPUs", ICPP'17.
 *   Citations "P:NN" are lines of the paper text;
 *   "R-n" are the readings listed in DESIGN.md sec. 3 where the paper is silent.
 *
 * One time step k is the paper's four-step loop:
 *   rp_deposit_step        1) particle deposition onto the N_X x N_Y grid D_k
 *   rp_compute_potentials  2) retarded potentials at every grid point, Eq. 1-2,
 *                             COMPUTE-POTENTIALS(k, V, tau, g, D) of Algorithm 1
 *   rp_compute_fields      3) self-fields from the potentials
 *   rp_push_particles      4) leap-frog Lorentz push by dt
 *
 * Conventions (all functions):
 *   - Array arguments are DEVICE pointers unless the name ends in _host.  The caller
 *     owns them; the library never frees caller memory and keeps no pointer to it
 *     after the call returns.  Device arrays must be 8-byte aligned.
 *   - All device work is ordered on the context's stream (rp_set_stream); calls
 *     return after enqueueing, except where "syncs" is stated.
 *   - Every call returns RP_OK (0) or a negative RP_E* code; no exception or exit()
 *     crosses the ABI.  rp_strerror() gives a static description, rp_last_error()
 *     the detailed message of the last failing call on that context.
 *   - FP64 everywhere (double-precision GFLOP/s).  Units are Gaussian with
 *     the caller's length/time units: phi = I_rho, A = I_{rho beta} (R-1).
 *   - One context per stream / host thread.  Contexts are independent: every entry point
 *     makes the context's device current and restores the caller's device before returning.
 *   - Multi-GPU: one process and one context per GPU, created with an rp_dist.
 *     Particles are sharded by the caller; the history ring is replicated; mesh points are
 *     sharded inside rp_compute_potentials.  The two exchanges of a step (the partial moment
 *     grids after deposition, the potential shards after integration) are NCCL all-gathers
 *     issued by librp on the context's stream, so every output covers the full mesh on every
 *     rank and the same calls serve N = 1 and N > 1.
 */
#ifndef RP_H_
#define RP_H_

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define RP_OK 0
#define RP_EINVAL (-1)  /* bad argument or configuration                      */
#define RP_ENOMEM (-2)  /* device or host allocation failed                    */
#define RP_ECUDA (-3)   /* CUDA runtime / kernel error (see rp_last_error)     */
#define RP_ENCCL (-4)   /* NCCL unavailable or a collective failed             */
#define RP_ESTATE (-5)  /* call out of order (e.g. potentials before deposit)  */
#define RP_ENODEV (-6)  /* no usable CUDA device                               */

#define RP_SRC_GRID 0   /* integrand from the deposited history (the product)  */
#define RP_SRC_GAUSS 1  /* analytic Gaussian sheet (test source)   */
#define RP_SRC_DISK 2   /* analytic uniform disk (test source)     */

typedef struct rp_ctx rp_ctx;

/* Grid frame of one time step: lab = O + u (c, s) + v (-s, c); grid node (ix, iy) sits
 * at local (ix*hx, iy*hy).  Frames move with the bunch (R-7). */
typedef struct {
  double ox, oy, cos_psi, sin_psi;
} rp_frame;

typedef struct {
  int32_t nx, ny;          /* grid nodes, >= 4 (P:32 N_X x N_Y); mesh points V = all nodes      */
  double hx, hy;           /* node spacing, > 0                                                  */
  int32_t history_depth;   /* kappa_max >= 1 subregions of reach; ring holds kappa_max+2 grids  */
  double c, dt;            /* > 0; subregion width c*dt (P:45 S_j = [j c dt, (j+1) c dt])        */
  double tau;              /* > 0; absolute tolerance per component (P:170 tau = 1e-6)           */
  int32_t n_theta;         /* even >= 2; inner Newton-Cotes panels per arc (R-11)          */
  int32_t max_depth;       /* 1..60 bisection cap of the outer tree (R-12)                       */
  int32_t n_root;          /* 2: roots are the two halves of each clipped S_j, and for the near
                              field S_0 the 2^L pieces no longer than max(nx hx, ny hy) / 8,
                              2 <= L <= 7 (R-12b); 1: [A, B] itself everywhere; 4: quarters
                              for j >= 1                                                      */
  int32_t device;          /* CUDA ordinal                                                       */
  int32_t outer_rule;      /* RP_RULE_GK15 (default, R-8) or RP_RULE_SIMPSON: the paper's own   */
                           /* rule (P:155 RP-QUADRULE), Boole value + |S2 - S1|/15 estimate (R-22) */
  int32_t interp;          /* spatial part of the "27 neighbouring points": RP_INTERP_TSC */
                           /* (default, R-6) or RP_INTERP_LAGRANGE3 (tri-quadratic Lagrange with  */
                           /* the time interpolation, R-25; discontinuous across cells; arc end  */
                           /* nodes on the support boundary take the outside limit 0, R-25b)     */
} rp_config;

#define RP_RULE_GK15 0
#define RP_RULE_SIMPSON 1
#define RP_INTERP_TSC 0
#define RP_INTERP_LAGRANGE3 1

typedef struct {
  int64_t n_lost;          /* particles whose 3x3 stencil leaves the grid (R-14)                 */
  double q_lost, q_total;
} rp_deposit_info;

typedef struct {
  int64_t evals;           /* integrand nodes f(r', theta', t') of the rules (as the oracle counts)*/
  int64_t nodes;           /* r' nodes (15 per GK15 segment)                                     */
  int64_t segments;        /* GK15 segments evaluated (sum of nseg)                              */
  int64_t leaves;          /* accepted segments                                                  */
  int64_t capped;          /* leaves accepted at max_depth with err > tol                        */
  int64_t ties;            /* decisions with |err - tol| / tol < 1e-9                            */
  int64_t items;           /* (point, subregion) pairs with support                              */
  int32_t max_level;       /* deepest tree level reached                                         */
  int32_t kappa;           /* subregions kappa(k) used at this step (R-3)                        */
  int64_t skipped;         /* of `evals`, arc end nodes on the support boundary, where the zero-
                              padded TSC integrand vanishes (DESIGN R-24) or the Lagrange-3 one
                              takes its outside limit 0 (R-25b), not evaluated; the evaluations
                              performed are evals - skipped                                     */
  int64_t units;           /* subtree work units walked separately (deep near-field trees split at
                              the work-split level, rp_set_work_split); 0 when off */
} rp_potential_info;

/* Multi-GPU membership of a context.  rank in [0, world).  Either nccl_comm is
 * an initialised ncclComm_t of `world` ranks whose rank `rank` uses cfg->device (caller-owned,
 * must outlive the context), or nccl_comm is NULL and nccl_id holds the bytes of one
 * ncclUniqueId obtained by rank 0 from rp_nccl_unique_id and broadcast by the caller to every
 * rank: rp_create then creates the communicator (collective: every rank must call it) and
 * rp_destroy frees it.  world = 1 is allowed (a one-rank communicator). */
#define RP_NCCL_ID_BYTES 128
typedef struct {
  int32_t rank, world;
  void* nccl_comm;
  unsigned char nccl_id[RP_NCCL_ID_BYTES];
} rp_dist;

/* Fill id_out with a fresh ncclUniqueId (call on one rank, broadcast the bytes).
 * ENCCL when NCCL cannot be loaded. */
int rp_nccl_unique_id(unsigned char id_out[RP_NCCL_ID_BYTES]);

/* Create a context on cfg->device: allocates the HBM history ring of history_depth+2
 * FP64 moment grids [slot][ny+6][nx+6][4] (zero-padded by 3 nodes) and scratch.
 * dist = NULL: single GPU.  dist != NULL: this process is rank dist->rank of dist->world
 * (see rp_dist); the NCCL communicator is created here when dist->nccl_comm is NULL.
 * EINVAL on an invalid config, ENODEV / ENOMEM / ECUDA on device failures, ENCCL when the
 * communicator cannot be created.  The caller's current device is left unchanged. */
int rp_create(const rp_config* cfg, const rp_dist* dist, rp_ctx** out);

/* Subtree work units: in the near-field subregion S_0 a segment at level
 * level-1 that splits hands its two children to a second, persistent launch instead of
 * descending (at most `budget` per item, the first in DFS order; a segment that would exceed
 * the budget descends in place), so one deep tree does not bound the step on one warp.  The
 * tree, every decision and the counts are unchanged; only the summation groups the subtrees
 * (results within rounding, bit-identical across ranks).  level = 0 turns it off; default
 * level 12, budget 64.  budget = 0 keeps the default.  EINVAL unless level == 0 or
 * 2 <= level <= max_depth, and budget == 0 or an even number in 2..64. */
int rp_set_work_split(rp_ctx* ctx, int32_t level, int32_t budget);

/* Destroy a context (NULL is ignored).  Synchronises its stream first. */
void rp_destroy(rp_ctx* ctx);

/* Use `stream` (a cudaStream_t; NULL = legacy default stream) for all later work. */
int rp_set_stream(rp_ctx* ctx, void* stream);

/* Optional pre-history, allowed only before the first deposit (else ESTATE).
 * n_pre in 1..history_depth+1 levels l = -n_pre .. -1; frames_host[n_pre] oldest first.
 * rigid = 0: grids_dev holds [n_pre][ny][nx][4] FP64 moment grids (component 3 ignored).
 * rigid = 1: grids_dev must be NULL; every pre-history level l receives the step-0 grid
 *            when the first deposit is appended (steady state): rho copied,
 *            the current rotated from frame 0 to frame l (J_l = R(psi_l - psi_0) J_0 with
 *            cos/sin of the difference from the frames' (cos, sin), R-23), so that every
 *            level holds the same comoving bunch.  Static frames: an exact copy.
 * Without pre-history, kappa(k) = min(kappa_max, k - 1) (R-3). */
int rp_history_init(rp_ctx* ctx, int32_t n_pre, const rp_frame* frames_host,
                    const double* grids_dev, int32_t rigid);

/* Bytes of one partial-deposit buffer (16-byte aligned device memory). */
int64_t rp_partial_bytes(const rp_ctx* ctx);

/* Partial deposition of n local particles (SoA x, y, u_x, u_y with u = gamma*beta) of
 * charge q each on frame_k (TSC, R-14) into partial_dev, an opaque buffer of
 * rp_partial_bytes() bytes holding the EXACT sums of (rho, rho*beta_x, rho*beta_y) per node:
 * each particle contribution is rounded once to 128-bit fixed point (quantum 2^-s with
 * 2^s ~ 2^85 (hx hy)/|q|), so sums do not depend on order or grouping.  Bins are computed
 * without FMA so they are bit-identical to the oracle (R-13).  Atomics-free: particles are
 * radix-sorted by bin and every node sums its 9 neighbour bins.  info (nullable) syncs. */
int rp_deposit(rp_ctx* ctx, const double* x, const double* y, const double* ux,
               const double* uy, double q, int64_t n, const rp_frame* frame_k,
               void* partial_dev, rp_deposit_info* info);

/* Advance to the next step k (0 at the first call) and store D_k = the exact sum of
 * n_parts consecutive partial buffers (e.g. all-gathered from the ranks), rounded once to
 * FP64, into ring slot k mod H with frame_k ("stored linearly on the device memory").
 * D_k is bit-identical for any split of the particles over ranks. */
int rp_history_append(rp_ctx* ctx, const void* partials_dev, int32_t n_parts,
                      const rp_frame* frame_k);

/* rp_deposit of this rank's particles into context scratch, then rp_history_append of the
 * partials of all ranks: with an rp_dist the partial buffers are all-gathered over NCCL on the
 * context's stream first (rank order), so D_k is identical on every rank and bit-identical to
 * a single-GPU deposit of all particles.  info (nullable, syncs) counts this rank's particles. */
int rp_deposit_step(rp_ctx* ctx, const double* x, const double* y, const double* ux,
                    const double* uy, double q, int64_t n, const rp_frame* frame_k,
                    rp_deposit_info* info);

/* Retarded potentials at all nx*ny nodes of the current frame (Eq. 1-2, Alg. 1).
 * With an rp_dist of world > 1 this rank integrates its share of the mesh points (dealt
 * longest-predicted-first over ranks from the previous step's counts, identical on every
 * rank) and the shards are all-gathered over NCCL, so the outputs cover the full mesh on
 * every rank; info then counts this rank's work only.  Enqueue-only: the call returns without
 * waiting for the device unless info is given (the work is capturable in a CUDA graph after
 * one warm-up call has sized the scratch).
 * For every (point p, subregion j < kappa(k)): support clip [A, B] of S_j (R-5), then a
 * deterministic top-down dyadic GK15 tree from the n_root halves of [A, B] (for the near
 * field j = 0 the pieces no longer than an eighth of the grid's extent, R-12b): accept a
 * segment iff max_c |K15_c - G7_c| <= tau (b - a) / R(p), R(p) = kappa(k) c dt, or at
 * max_depth (R-8..R-12).  Work items are scheduled longest-predicted-first from the
 * previous step's per-(p, j) segment counts (the paper's forecast g, used for
 * scheduling only).  Outputs [ny*nx] (flattened iy*nx + ix): phi = sum K_0,
 * ax = sum K_1, ay = sum K_2, err = sum of leaf errors, nseg = segments evaluated.
 * err / nseg may be NULL.  info (nullable) syncs. */
int rp_compute_potentials(rp_ctx* ctx, double* phi, double* ax, double* ay, double* err,
                          int32_t* nseg, rp_potential_info* info);

/* As rp_compute_potentials but only for the points owned by `rank` of `world` under the
 * context's shard map (mesh-point data parallelism): points are dealt
 * longest-predicted-first in a snake order over ranks from the previous step's counts,
 * identical on every rank.  Writes shard_out [cap][6] FP64 records
 * (point id, phi, ax, ay, err, nseg) for the owned points, rows >= *n_out zero-filled;
 * cap >= rp_shard_capacity().  Combine the all-gathered shards with rp_shard_scatter. */
int rp_compute_potentials_shard(rp_ctx* ctx, int32_t rank, int32_t world, double* shard_out,
                                int64_t cap, int64_t* n_out, rp_potential_info* info);

/* Rows per shard buffer: ceil(nx*ny / world). */
int64_t rp_shard_capacity(const rp_ctx* ctx, int32_t world);

/* Scatter `world` gathered shard buffers [world][cap][6] into full-mesh outputs and
 * record the counts for the next step's schedule (identical on every rank). */
int rp_shard_scatter(rp_ctx* ctx, const double* shards, int32_t world, int64_t cap,
                     double* phi, double* ax, double* ay, double* err, int32_t* nseg);

/* Self-fields on mesh k (R-15, R-15b): second-order central differences (one-sided at
 * the edges) in frame coordinates rotated to the lab;
 *   E = -grad phi - (1/c) dA/dt,  B_z = d_x A_y - d_y A_x,
 *   dA/dt = (1/dt) sum_j BD_j A_{k-j} - (V . grad) A_k,  V = (1/dt) sum_j BD_j P_{k-j},
 * consistent order-m backward differences at t_k of the node values and of the node position
 * on the frames of levels k .. k-m (exact for a field at rest in the lab, O(dt^m) for one
 * co-moving with the mesh).  a_prev: DEVICE [n_prev][2][ny*nx], (A_x, A_y) of steps k-1, ...,
 * k-n_prev (most recent first); n_prev = 0..4 (0: dA/dt omitted); m = n_prev, lowered when the
 * ring holds fewer frames.  All other arrays [ny*nx].  EINVAL on n_prev outside 0..4. */
int rp_compute_fields(rp_ctx* ctx, const double* phi, const double* ax, const double* ay,
                      const double* a_prev, int32_t n_prev, double* ex, double* ey, double* bz);

/* Relativistic Boris leap-frog push by dt (R-15) of n particles in place:
 * TSC gather of (E_x, E_y, B_z) on frame k (same weights as deposition), plus a uniform
 * external B_z = bz_ext; du/dt = q_over_mc (E + beta x B); x += c dt u / gamma. */
int rp_push_particles(rp_ctx* ctx, double* x, double* y, double* ux, double* uy, int64_t n,
                      double q_over_mc, double bz_ext, const double* ex, const double* ey,
                      const double* bz);

/* Lorentz force per unit charge on n particles, F = E + beta x (B_z + bz_ext) z-hat (lab x, y
 * components), from the same TSC gather of (E_x, E_y, B_z) on frame k as rp_push_particles
 * (R-15): the particle-level forces F_i of the paper's validation (Fig. 2-3).
 * beta = u / sqrt(1 + u^2).  fx, fy [n] DEVICE outputs. */
int rp_particle_forces(rp_ctx* ctx, const double* x, const double* y, const double* ux,
                       const double* uy, int64_t n, double bz_ext, const double* ex,
                       const double* ey, const double* bz, double* fx, double* fy);

/* Time-centred momenta for the deposit's current (R-27): the leap-frog momenta u (at
 * t_k - dt/2) advanced by frac * dt in the uniform external B_z = bz_ext (the Boris
 * rotation of rp_push_particles with E = 0), written to ux_out / uy_out [n] (DEVICE; may alias
 * the inputs).  The loop deposits with frac = 1/2 so the current of step k is rho v(t_k); a
 * current half a step behind the bunch's motion is misaligned by half the step's bend angle,
 * which swamps the CSR force (a 1e-4 residual of space-charge-sized terms). */
int rp_kick_external(rp_ctx* ctx, const double* ux, const double* uy, int64_t n,
                     double q_over_mc, double bz_ext, double frac, double* ux_out,
                     double* uy_out);

/* One whole step through HOST buffers (end-to-end path).  With an rp_dist the host arrays
 * hold this rank's particle shard and the mesh outputs are the full mesh.  Copies the particles
 * host->device, runs kick_external (frac 1/2) + deposit_step, compute_potentials,
 * compute_fields (with the previous
 * steps' A kept by the context, up to 4), push, and copies the pushed particles and the six mesh
 * outputs back.  x_host .. uy_host are updated in place; mesh_host is [6][ny*nx]
 * (phi, ax, ay, ex, ey, bz).  Pinned host memory gives full-bandwidth copies.  info
 * (nullable) receives the potentials' work counters.  Syncs. */
int rp_step_host(rp_ctx* ctx, double* x_host, double* y_host, double* ux_host,
                 double* uy_host, int64_t n, double q, const rp_frame* frame_k,
                 double q_over_mc, double bz_ext, double* mesh_host, rp_potential_info* info);

/* ---- state access (checkpoint / parity from a common seeded state) ---- */

/* Overwrite the whole history: step index k, pre-history depth n_pre (for kappa(k)),
 * frames_host[H] and ring_dev [H][ny][nx][4] in ring-slot order (slot = level mod H).
 * Clears the schedule forecast.  Allowed at any time. */
int rp_load_state(rp_ctx* ctx, int32_t k, int32_t n_pre, const rp_frame* frames_host,
                  const double* ring_dev);

/* Copy the ring out ([H][ny][nx][4], unpadded) and/or the frames; NULLs skip.  Syncs. */
int rp_save_state(rp_ctx* ctx, int32_t* k_out, double* ring_dev, rp_frame* frames_host);

/* Bin index of every particle of the last rp_deposit (-1 = lost), [n]. */
int rp_debug_bins(rp_ctx* ctx, int32_t* bins_dev, int64_t n);

/* The support clip of the last rp_compute_potentials call (step a5, R-5: per (point p,
 * subregion j) the r'-interval [A, B] of S_j where the circle about p meets the support
 * rectangle at the retarded time, by 64-step bisection on squared distances): copies
 * npts * kappa_max pairs (A, B), p-major, into ab_dev (DEVICE, caller-owned, 2 * n doubles
 * with n = nx * ny * history_depth); (0, 0) for items without support or with j >= kappa.
 * The arithmetic mirrors the oracle's operation order with IEEE round-to-nearest intrinsics,
 * so the limits are bit-identical to it.  RP_ESTATE before the first potentials call. */
int rp_debug_clip(rp_ctx* ctx, double* ab_dev, int64_t n);

/* Per-point (nleaf, capped) of the last rp_compute_potentials call (the 7-tuple of P:110
 * beside phi, A, err and nseg): accepted segments and the leaves accepted
 * at max_depth with err > tol, summed over the point's subregions; int32 DEVICE arrays of
 * n = nx*ny entries (either may be NULL).  Points not owned by the last shard call keep
 * stale values.  EINVAL on a wrong n, ESTATE before the first potentials call. */
int rp_debug_point_counts(rp_ctx* ctx, int32_t* nleaf_dev, int32_t* capped_dev, int64_t n);
/* Accepted segments of every (point, subregion) item of the last rp_compute_potentials (the
 * observed access pattern n_j(p) of P:83-95 that the forecast reads), uint16 (saturating)
 * [nx * ny][history_depth] device array, n = nx * ny * history_depth.  Enqueue-only. */
int rp_debug_item_leaves(rp_ctx* ctx, uint16_t* leaves_dev, int64_t n);

/* Test hook: potentials with an analytic source in place of the grid:
 * kind = RP_SRC_GAUSS (centre (x0,y0) frame-local, width = sigma, q = Q) or RP_SRC_DISK
 * (width = radius, q = surface density); (bx, by) = beta; amp_host[H] per-slot amplitudes
 * (NULL = 1).  Same clip / tree / inner rule / kernels as the grid path. */
int rp_debug_potentials_analytic(rp_ctx* ctx, int32_t kind, double x0, double y0,
                                 double width, double q, double bx, double by,
                                 const double* amp_host, double* phi, double* ax, double* ay,
                                 double* err, int32_t* nseg, rp_potential_info* info);

/* Work-scheduling forecast (the paper's predictor g, used ONLY to order work; the
 * results are bit-identical for every policy, R-17):
 *   RP_SCHED_INDEX        no forecast: (point, subregion) items in index order;
 *   RP_SCHED_PERSISTENCE  (default) predicted cost of (p, j) = segments it took last step;
 *   RP_SCHED_KNN          kNN regression over mesh points: predicted cost of (p, j) =
 *                         mean of last step's cost of (q, j) over the k nearest mesh points q
 *                         of the comoving mesh (k in {1, 5, 9, 25}; 1 = persistence).
 *   RP_SCHED_SUBREGION    persistence forecast, items ordered subregion-major (j ascending) and
 *                         longest-predicted-first within each subregion, so the warps running
 *                         at any moment share one subregion's three history levels (L2 reuse
 *                         when the ring is larger than L2, configs 4-5).
 * Items are then run longest-predicted-first (LPT). */
#define RP_SCHED_INDEX 0
#define RP_SCHED_PERSISTENCE 1
#define RP_SCHED_KNN 2
#define RP_SCHED_SUBREGION 3
int rp_set_schedule(rp_ctx* ctx, int32_t policy, int32_t k);

/* Predictive-RP variant: the paper's own COMPUTE-POTENTIALS (Algorithm 1; DESIGN
 * reading R-26) instead of the canonical dyadic tree.  At every step that has the previous
 * step's observed access pattern n_j(p) (accepted segments per point and subregion, recorded
 * by every rp_compute_potentials call), the forecast partition is built on the host (the
 * paper's lines 1-12 run on the CPU too): line 3 kNN forecast of n_j(p) over the
 * k nearest mesh nodes (k in {1, 5, 9, 25}, as rp_set_schedule); line 4 uniform
 * partitioning of each subregion S_j into n_j(p) pieces; line 6 k-means of the
 * pattern vectors into n_clusters clusters (0: max(nx, ny); deterministic centres
 * and Lloyd passes, at most max_iters); lines 9-12 MERGE-LISTS of the partitions of each
 * cluster.  The kernel then integrates each (point, subregion) item over its cluster's
 * merged intervals cut to the item's support (lines 13-16), each interval being the root
 * of an adaptive dyadic tree that refines it where the estimate misses the tolerance
 * (lines 18-24).  Results differ from the canonical tree within tau and depend on the
 * forecast.  A step without a previous pattern uses the canonical tree.
 * Single-GPU path only: rp_compute_potentials_shard, and rp_compute_potentials on a context
 * with world > 1, return RP_EINVAL while enabled.
 * enable = 0 restores the canonical tree.  Returns RP_EINVAL on a bad k or n_clusters < 0. */
int rp_set_predictive(rp_ctx* ctx, int32_t enable, int32_t knn, int32_t n_clusters,
                      int32_t max_iters);

/* Line 4 of the Predictive-RP variant: RP_PART_UNIFORM (default) cuts S_j into
 * n_j(p) equal pieces; RP_PART_ADAPTIVE refines the partition accepted at the earlier
 * step (DESIGN reading R-26b): each of the d_j pieces the item (p, j) was integrated on
 * in the previous rp_compute_potentials is cut into max(1, round(n_j / d_j)) equal pieces,
 * a_j and b_j close the list, an item without an earlier partition falls back to uniform
 * partitioning; then MERGE-LISTS as before.  With ADAPTIVE every call records its accepted
 * leaves on the device (one 32-B record per leaf, a buffer of max(2^22, 4 x nx x ny x
 * history_depth) records, grown to 4x the previous call's leaves when they fill half of it and to
 * 2x the count after an overflow; a call whose predecessor overflowed it uses uniform
 * partitioning, reported as partition = -1).  EINVAL on another mode, ENOMEM when the buffer cannot be
 * allocated.  Takes effect at the next rp_compute_potentials. */
#define RP_PART_UNIFORM 0
#define RP_PART_ADAPTIVE 1
int rp_set_predictive_partition(rp_ctx* ctx, int32_t mode);

typedef struct {
  int32_t active;          /* 1 if the last rp_compute_potentials used a forecast partition    */
  int32_t clusters;        /* k-means clusters m                                               */
  int32_t kmeans_passes;   /* assignment passes made                                           */
  int32_t partition;       /* line 4 used: RP_PART_UNIFORM / RP_PART_ADAPTIVE, or -1 when
                              adaptive was asked for but the earlier leaves overflowed        */
  int64_t breakpoints;     /* total length of the merged partition lists                      */
  double host_ms;          /* host time of lines 1-12 (download of n_j, forecast, clustering,  */
                           /* merge, upload), included in the call                             */
} rp_predictive_info;
/* Statistics of the last rp_compute_potentials (host struct, no sync).  clusters_host
 * (nullable): the k-means cluster of every mesh point [nx * ny] (parity with the oracle). */
int rp_predictive_info_read(rp_ctx* ctx, rp_predictive_info* out, int32_t* clusters_host);
/* The merged partition lists of the last call that used a forecast (host copies; parity with
 * the oracle's MERGE-LISTS): off_host [clusters * history_depth + 1] (nullable), bp_host
 * [breakpoints] (nullable).  ESTATE when no call has used a forecast partition. */
int rp_predictive_lists_read(rp_ctx* ctx, int64_t* off_host, double* bp_host);

/* Per-kernel device time, measured with CUDA events recorded on the context's stream around
 * each launch while profiling is enabled (bench.py's live roofline numbers). */
typedef struct {
  double deposit_ms;       /* bin + sort + gather + node sums                                   */
  double append_ms;        /* rank-order sum into the ring                                      */
  double clip_ms;          /* support clip + schedule keys                                      */
  double sort_ms;          /* schedule sort (CUB)                                               */
  double integrate_ms;     /* the GK15 integrator (dominant kernel): items + subtree units + merge */
  double reduce_ms;        /* per-point reduction                                               */
  double fields_ms;
  double push_ms;
  int64_t integrate_launches;  /* integrator calls (each: the item launch, then the units')  */
  double units_ms;         /* of integrate_ms: the subtree-unit launch, its sort and merge      */
  double step_ms;          /* rp_step_host: its device part, deposit through push (the copies
                              before and after it excluded)                                     */
} rp_profile;

/* enable != 0 starts (and resets) event timing; 0 stops it.  Adds two event records per
 * instrumented launch; off by default. */
int rp_profile_enable(rp_ctx* ctx, int32_t enable);

/* Sum of the recorded device times since the last enable.  Syncs the stream. */
int rp_profile_read(rp_ctx* ctx, rp_profile* out);

/* Number of kernel launches this context has issued (for bench.py's gpu_launches). */
int64_t rp_launch_count(const rp_ctx* ctx);

/* Static text for an RP_E* code. */
const char* rp_strerror(int code);

/* Detailed message of the last failing call on ctx (never NULL). */
const char* rp_last_error(const rp_ctx* ctx);

/* ABI version (major*100 + minor). */
int rp_version(void);

#ifdef __cplusplus
}
#endif
#endif /* RP_H_ */
