// rp_internal.cuh -- context and shared device helpers of librp (product path).
// Nothing here is shared with oracle/ (test infrastructure): the two are written
// independently from PAPER.md and DESIGN.md's readings.
#pragma once

#include <cuda_runtime.h>
#include <nccl.h>
#include <stdint.h>
#include <string.h>

#include <string>
#include <vector>

#include "../../include/rp.h"

#define RP_PAD 3  // zero border (nodes) around every ring grid: stencils never bounds-check
#define RP_NCCL_ID_BYTES 128

// NCCL entry points, resolved at run time (nccl_dyn.cu)
struct RpNccl {
  void* handle;
  ncclResult_t (*get_unique_id)(ncclUniqueId*);
  ncclResult_t (*comm_init_rank)(ncclComm_t*, int, ncclUniqueId, int);
  ncclResult_t (*comm_destroy)(ncclComm_t);
  ncclResult_t (*all_gather)(const void*, void*, size_t, ncclDataType_t, ncclComm_t,
                             cudaStream_t);
  const char* (*error_string)(ncclResult_t);
  ncclResult_t (*get_version)(int*);
};
const RpNccl* rp_nccl_api(std::string* err);

// Makes the context's device current for the duration of an entry point and restores the
// caller's device on exit (contexts on different GPUs in one process stay independent).
struct DeviceGuard {
  int prev = -1, dev;
  explicit DeviceGuard(int d) : dev(d) {
    if (cudaGetDevice(&prev) != cudaSuccess) prev = -1;
    if (prev != dev) cudaSetDevice(dev);
  }
  ~DeviceGuard() {
    if (prev >= 0 && prev != dev) cudaSetDevice(prev);
  }
};

struct rp_ctx {
  rp_config cfg;
  int H = 0;                 // ring slots = history_depth + 2
  int PX = 0, PY = 0;        // padded grid dims (nx + 6, ny + 6)
  size_t slot_doubles = 0;   // PX * PY * 4
  cudaStream_t stream = 0;
  int sm_count = 0;

  // multi-GPU (rp_dist): mesh points sharded over `world` ranks, history
  // replicated; the two exchanges of a step are NCCL all-gathers on `stream`
  int dist_on = 0, rank = 0, world = 1;
  ncclComm_t comm = nullptr;
  int own_comm = 0;                 // created by rp_create (destroyed by rp_destroy)
  unsigned char* partials_all = nullptr;  // [world][rp_partial_bytes]
  double* shard_buf = nullptr;      // [shard_cap][6] this rank's potential shard
  double* shards_all = nullptr;     // [world][shard_cap][6]
  int64_t shard_cap = 0;

  // history: ring [H][PY][PX][4] FP64 and frames [H]
  double* ring = nullptr;
  rp_frame* frames_dev = nullptr;
  rp_frame* fh = nullptr;    // host copy of frames [H]
  int k = -1;                // current step (-1 before the first append)
  int n_pre = 0;             // pre-history levels available below step 0
  int rigid_pending = 0;     // rigid pre-history: fill on first append
  int prehist_set = 0;

  // deposition scratch (grown on demand)
  int64_t dep_cap = 0;
  int32_t* keys = nullptr;      // bin per particle (nx*ny for lost)
  int32_t* keys_sorted = nullptr;
  int32_t* perm = nullptr;      // particle index
  int32_t* perm_sorted = nullptr;
  double4* rec = nullptr;       // (dx, dy, bx, by) per particle
  double4* rec_sorted = nullptr;
  int32_t* bin_start = nullptr; // [nx*ny + 1]
  int64_t last_n = 0;
  void* partial = nullptr;      // exact partial buffer (rp_partial_bytes) for rp_deposit_step
  void* cub_tmp = nullptr;
  size_t cub_tmp_bytes = 0;

  // potentials scratch: dense (point, subregion) arrays of npts * kappa_max
  double2* clipAB = nullptr;        // [A, B] per (p, j)
  uint32_t* sched_key = nullptr;    // sort keys (0xFFFFFFFF = empty)
  uint32_t* sched_key_sorted = nullptr;
  int32_t* sched_idx = nullptr;     // iota
  int32_t* sched_order = nullptr;   // sorted item ids (p * kappa_max + j)
  uint16_t* cost_prev = nullptr;    // forecast: previous step's segments per (p, j)
  double4* item_val = nullptr;      // (phi, ax, ay, err) per (p, j)
  int4* item_cnt = nullptr;         // (nseg, nleaf, capped, ties) per (p, j)
  uint2* item_aux = nullptr;        // (max_level, evals) per (p, j)
  unsigned long long* counters = nullptr;  // [16] device counters
  double* amp_dev = nullptr;        // [H] analytic amplitudes
  double2* trig_full = nullptr;     // [n_theta] (cos, sin)(2 pi m / n_theta)
  int has_forecast = 0;
  int sched_policy = 1;             // RP_SCHED_*
  int sched_k = 9;                  // kNN neighbours

  // Predictive-RP variant (rp_set_predictive, DESIGN R-26)
  int pred_on = 0, pred_knn = 9, pred_m = 0, pred_iters = 20;
  uint16_t* leaves_prev = nullptr;  // [npts * kappa_max] accepted segments of the last call
  int have_leaves = 0;
  int32_t* cluster_dev = nullptr;   // [npts] k-means cluster of every point
  int64_t* bp_off_dev = nullptr;    // [m * kappa_max + 1] merged-list offsets
  double* bp_dev = nullptr;         // merged breakpoints
  int64_t bp_cap = 0, off_cap = 0;
  std::vector<int32_t> cluster_host;
  rp_predictive_info pred_info{};
  // adaptive partitioning (rp_set_predictive_partition, R-26b): accepted leaves of the last
  // call, (a, b, item, 0) per leaf, appended by k_integrate; the count lives apart from the
  // per-call counters so the next call can read it before they are cleared
  int pred_part = 0;
  double4* leaf_rec = nullptr;
  long long leaf_cap = 0;
  unsigned long long* leaf_count_dev = nullptr;
  int leaf_valid = 0;               // the last call recorded its leaves
  std::vector<int64_t> pred_off_host;  // the last merged lists (rp_predictive_lists_read)
  std::vector<double> pred_bp_host;

  // subtree work units of the deep trees (k_integrate split_level; rp_set_work_split)
  int split_level = 12;             // 0 = off
  int unit_budget = 64;             // units per near-field item (<= the slots allocated, 64)
  int split_j = 1;                  // split the trees of subregions j < split_j (the near field)
  long long unit_slots = 0;         // npts * split_j * unit budget
  int32_t* unit_ndef = nullptr;     // [npts * split_j] units deferred per near-field item
  unsigned long long* unit_key = nullptr;
  unsigned long long* unit_okey = nullptr;  // launch-order keys of the slots
  unsigned long long* unit_okey_sorted = nullptr;
  int32_t* unit_iota = nullptr;
  int32_t* unit_perm = nullptr;
  double4* unit_val = nullptr;
  int4* unit_cnt = nullptr;
  uint2* unit_aux = nullptr;

  // sharding scratch
  int32_t* point_key = nullptr;     // per point predicted work key
  int32_t* point_key_sorted = nullptr;
  int32_t* point_idx = nullptr;
  int32_t* point_order = nullptr;
  int32_t* point_owner = nullptr;   // rank owning each point
  int32_t* nseg_prev_pt = nullptr;  // per point segments of the last step (shard map)
  int2* point_cnt = nullptr;        // per point (leaves, capped) of the last call

  // end-to-end (host buffer) path scratch
  int64_t host_cap = 0;
  double* hx_d = nullptr; double* hy_d = nullptr; double* hux_d = nullptr; double* huy_d = nullptr;
  double* cux_d = nullptr; double* cuy_d = nullptr;  // time-centred momenta of the deposit (R-27)
  double* mesh_d = nullptr;         // [6][npts]: phi ax ay ex ey bz of the last rp_step_host
  double* aprev_d = nullptr;        // [4][2][npts]: A of the 4 steps before (most recent first)
  int n_prev_A = 0;                 // how many of them are valid

  int64_t launches = 0;
  std::string err;

  // event timing (rp_profile_enable / rp_profile_read)
  struct ProfRec { int kind; cudaEvent_t a, b; };
  int prof_on = 0;
  std::vector<ProfRec> prof;
  std::vector<cudaEvent_t> ev_pool;
  double prof_acc[10] = {0, 0, 0, 0, 0, 0, 0, 0, 0, 0};
  int64_t prof_integrate_launches = 0;
};

enum { PK_DEPOSIT = 0, PK_APPEND, PK_CLIP, PK_SORT, PK_INTEGRATE, PK_REDUCE, PK_FIELDS, PK_PUSH,
       PK_UNITS, PK_STEP };

static inline cudaEvent_t prof_event(rp_ctx* ctx) {
  if (!ctx->ev_pool.empty()) {
    cudaEvent_t e = ctx->ev_pool.back();
    ctx->ev_pool.pop_back();
    return e;
  }
  cudaEvent_t e = nullptr;
  cudaEventCreate(&e);
  return e;
}

// RAII: records an event pair around the enclosed launches when profiling is on
struct ProfScope {
  rp_ctx* ctx;
  int kind;
  cudaEvent_t a = nullptr;
  ProfScope(rp_ctx* c, int k) : ctx(c), kind(k) {
    if (ctx->prof_on) {
      a = prof_event(ctx);
      cudaEventRecord(a, ctx->stream);
    }
  }
  ~ProfScope() {
    if (a) {
      cudaEvent_t b = prof_event(ctx);
      cudaEventRecord(b, ctx->stream);
      ctx->prof.push_back({kind, a, b});
      if (kind == PK_INTEGRATE) ctx->prof_integrate_launches++;
    }
  }
};

// ---------------------------------------------------------------- error helpers
#define RP_CUDA(call)                                                            \
  do {                                                                           \
    cudaError_t e_ = (call);                                                     \
    if (e_ != cudaSuccess) {                                                     \
      ctx->err = std::string(#call) + ": " + cudaGetErrorString(e_);             \
      return e_ == cudaErrorMemoryAllocation ? RP_ENOMEM : RP_ECUDA;             \
    }                                                                            \
  } while (0)

#define RP_CHECK_LAUNCH()                                                        \
  do {                                                                           \
    ctx->launches++;                                                             \
    cudaError_t e_ = cudaGetLastError();                                         \
    if (e_ != cudaSuccess) {                                                     \
      ctx->err = std::string("kernel launch: ") + cudaGetErrorString(e_);        \
      return RP_ECUDA;                                                           \
    }                                                                            \
  } while (0)

static inline int rp_fail(rp_ctx* ctx, int code, const char* msg) {
  if (ctx) ctx->err = msg;
  return code;
}

static inline int slot_of(int level, int H) { return ((level % H) + H) % H; }
__device__ __forceinline__ int slot_of_dev(int level, int H) { return ((level % H) + H) % H; }

static inline int kappa_of(const rp_ctx* ctx) {
  int kap = ctx->k + ctx->n_pre - 1;
  if (kap > ctx->cfg.history_depth) kap = ctx->cfg.history_depth;
  if (kap < 0) kap = 0;
  return kap;
}

// internal entry points implemented in the .cu files
int rp_deposit_impl(rp_ctx* ctx, const double* x, const double* y, const double* ux,
                    const double* uy, double q, int64_t n, const rp_frame* frame_k,
                    void* partial_dev, rp_deposit_info* info);
int rp_append_impl(rp_ctx* ctx, const void* partials, int32_t n_parts, const rp_frame* fk);
int64_t rp_partial_bytes_impl(const rp_ctx* ctx);
int rp_potentials_impl(rp_ctx* ctx, int src_kind, const double src[6], int32_t rank,
                       int32_t world, double* phi, double* ax, double* ay, double* err,
                       int32_t* nseg, double* shard_out, int64_t cap, int64_t* n_out,
                       rp_potential_info* info);
int rp_fields_impl(rp_ctx* ctx, const double* phi, const double* ax, const double* ay,
                   const double* a_prev, int n_prev, double* ex, double* ey, double* bz);
int rp_push_impl(rp_ctx* ctx, double* x, double* y, double* ux, double* uy, int64_t n,
                 double qmc, double bz_ext, const double* ex, const double* ey,
                 const double* bz);
int rp_forces_impl(rp_ctx* ctx, const double* x, const double* y, const double* ux,
                   const double* uy, int64_t n, double bz_ext, const double* ex, const double* ey,
                   const double* bz, double* fx, double* fy);
int rp_kick_impl(rp_ctx* ctx, const double* ux, const double* uy, int64_t n, double qmc,
                 double bz_ext, double frac, double* ox, double* oy);
int rp_scatter_impl(rp_ctx* ctx, const double* shards, int32_t world, int64_t cap,
                    double* phi, double* ax, double* ay, double* err, int32_t* nseg);
int rp_alloc_potential_scratch(rp_ctx* ctx);
int rp_predictive_setup(rp_ctx* ctx, int kap);
