// rp_api.cu -- the C ABI of librp (include/rp.h): context, history ring, state access and
// the argument checking around the kernels of deposit.cu, potentials.cu, fields_push.cu.
#include <new>

#include <algorithm>

#include "rp_internal.cuh"

// every entry point: a context, and its device current for the call (restored on return)
#define RP_ENTER(ctx)          \
  if (!(ctx)) return RP_EINVAL; \
  DeviceGuard device_guard_((ctx)->cfg.device)

namespace {

int validate(const rp_config* c) {
  if (!c) return RP_EINVAL;
  if (c->nx < 4 || c->ny < 4 || (int64_t)c->nx * c->ny > (1LL << 30)) return RP_EINVAL;
  if (!(c->hx > 0) || !(c->hy > 0) || !(c->c > 0) || !(c->dt > 0) || !(c->tau > 0)) return RP_EINVAL;
  if (c->history_depth < 1 || c->history_depth > 1000000) return RP_EINVAL;
  if ((int64_t)c->nx * c->ny * c->history_depth > 0x7fffffffLL) return RP_EINVAL;
  if (c->n_theta < 2 || (c->n_theta & 1) || c->n_theta > 4096) return RP_EINVAL;
  if (c->max_depth < 1 || c->max_depth > 60) return RP_EINVAL;
  if (c->n_root != 1 && c->n_root != 2 && c->n_root != 4) return RP_EINVAL;
  if (c->outer_rule != RP_RULE_GK15 && c->outer_rule != RP_RULE_SIMPSON) return RP_EINVAL;
  if (c->interp != RP_INTERP_TSC && c->interp != RP_INTERP_LAGRANGE3) return RP_EINVAL;
  return RP_OK;
}

__global__ void k_unpad(int nx, int ny, int PX, const double* __restrict__ slot,
                        double* __restrict__ out) {
  int id = blockIdx.x * blockDim.x + threadIdx.x;
  if (id >= nx * ny) return;
  int ix = id % nx, iy = id / nx;
  const double* s = slot + 4 * ((size_t)(iy + RP_PAD) * PX + (ix + RP_PAD));
  double* d = out + 4 * (size_t)id;
  d[0] = s[0]; d[1] = s[1]; d[2] = s[2]; d[3] = s[3];
}

__global__ void k_pad(int nx, int ny, int PX, const double* __restrict__ in,
                      double* __restrict__ slot) {
  int id = blockIdx.x * blockDim.x + threadIdx.x;
  if (id >= nx * ny) return;
  int ix = id % nx, iy = id / nx;
  const double* s = in + 4 * (size_t)id;
  double* d = slot + 4 * ((size_t)(iy + RP_PAD) * PX + (ix + RP_PAD));
  d[0] = s[0]; d[1] = s[1]; d[2] = s[2]; d[3] = 0.0;
}

__global__ void k_bins_out(int64_t n, int nbins, const int32_t* __restrict__ keys,
                           int32_t* __restrict__ out) {
  int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (i < n) out[i] = keys[i] == nbins ? -1 : keys[i];
}

void free_all(rp_ctx* c) {
  void* ptrs[] = {c->ring, c->frames_dev, c->keys, c->keys_sorted, c->perm, c->perm_sorted,
                  c->rec, c->rec_sorted, c->bin_start, c->partial, c->cub_tmp, c->clipAB,
                  c->sched_key, c->sched_key_sorted, c->sched_idx, c->sched_order, c->cost_prev,
                  c->item_val, c->item_cnt, c->item_aux, c->counters, c->amp_dev, c->trig_full,
                  c->point_key, c->point_key_sorted, c->point_idx, c->point_order,
                  c->point_owner, c->nseg_prev_pt, c->point_cnt, c->hx_d, c->hy_d, c->hux_d, c->huy_d, c->cux_d, c->cuy_d,
                  c->mesh_d, c->aprev_d, c->leaves_prev, c->cluster_dev, c->bp_off_dev, c->bp_dev,
                  c->unit_key, c->unit_okey, c->unit_okey_sorted, c->unit_iota, c->unit_perm, c->unit_val,
                  c->unit_ndef, c->partials_all, c->shard_buf, c->shards_all,
                  c->unit_cnt, c->unit_aux, c->leaf_rec, c->leaf_count_dev};
  for (void* p : ptrs)
    if (p) cudaFree(p);
  for (auto& r : c->prof) {
    cudaEventDestroy(r.a);
    cudaEventDestroy(r.b);
  }
  for (auto e : c->ev_pool) cudaEventDestroy(e);
  delete[] c->fh;
  if (c->comm && c->own_comm) {
    if (const RpNccl* api = rp_nccl_api(nullptr)) api->comm_destroy(c->comm);
  }
  c->comm = nullptr;
}

__global__ void k_point_counts(int64_t n, const int2* __restrict__ pc, int32_t* __restrict__ nleaf,
                               int32_t* __restrict__ capped) {
  int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (i >= n) return;
  if (nleaf) nleaf[i] = pc[i].x;
  if (capped) capped[i] = pc[i].y;
}

// NCCL all-gather of `bytes` per rank on the context's stream (rank order in recv)
int allgather(rp_ctx* ctx, const void* send, void* recv, size_t bytes) {
  std::string e;
  const RpNccl* api = rp_nccl_api(&e);
  if (!api) return rp_fail(ctx, RP_ENCCL, e.c_str());
  ncclResult_t r = api->all_gather(send, recv, bytes, ncclUint8, ctx->comm, ctx->stream);
  if (r != ncclSuccess) {
    ctx->err = std::string("ncclAllGather: ") + api->error_string(r);
    return RP_ENCCL;
  }
  return RP_OK;
}

// deposit of this rank's particles + (dist) all-gather of the partials + append
int deposit_step(rp_ctx* ctx, const double* x, const double* y, const double* ux,
                 const double* uy, double q, int64_t n, const rp_frame* fk, rp_deposit_info* info) {
  int rc = rp_deposit_impl(ctx, x, y, ux, uy, q, n, fk, ctx->partial, info);
  if (rc) return rc;
  if (!ctx->dist_on) return rp_append_impl(ctx, ctx->partial, 1, fk);
  if (!fk) return rp_fail(ctx, RP_EINVAL, "deposit_step: no frame");
  rc = allgather(ctx, ctx->partial, ctx->partials_all, (size_t)rp_partial_bytes_impl(ctx));
  if (rc) return rc;
  return rp_append_impl(ctx, ctx->partials_all, ctx->world, fk);
}

// potentials on the full mesh: single call, or (dist) this rank's shard + all-gather + scatter
int potentials_full(rp_ctx* ctx, double* phi, double* ax, double* ay, double* err, int32_t* nseg,
                    rp_potential_info* info) {
  if (!ctx->dist_on)
    return rp_potentials_impl(ctx, RP_SRC_GRID, nullptr, 0, 1, phi, ax, ay, err, nseg, nullptr, 0,
                              nullptr, info);
  if (ctx->pred_on) return rp_fail(ctx, RP_EINVAL, "potentials: Predictive-RP is single-GPU only");
  if (!phi || !ax || !ay) return rp_fail(ctx, RP_EINVAL, "potentials: null output");
  int rc = rp_potentials_impl(ctx, RP_SRC_GRID, nullptr, ctx->rank, ctx->world, nullptr, nullptr,
                              nullptr, nullptr, nullptr, ctx->shard_buf, ctx->shard_cap, nullptr,
                              info);
  if (rc) return rc;
  rc = allgather(ctx, ctx->shard_buf, ctx->shards_all, (size_t)ctx->shard_cap * 6 * sizeof(double));
  if (rc) return rc;
  return rp_scatter_impl(ctx, ctx->shards_all, ctx->world, ctx->shard_cap, phi, ax, ay, err, nseg);
}

}  // namespace

extern "C" {

int rp_version(void) { return 200; }

const char* rp_strerror(int code) {
  switch (code) {
    case RP_OK: return "ok";
    case RP_EINVAL: return "invalid argument or configuration";
    case RP_ENOMEM: return "out of memory";
    case RP_ECUDA: return "CUDA error";
    case RP_ENCCL: return "NCCL unavailable or a collective failed";
    case RP_ESTATE: return "call out of order";
    case RP_ENODEV: return "no usable CUDA device";
    default: return "unknown error";
  }
}

const char* rp_last_error(const rp_ctx* ctx) { return ctx ? ctx->err.c_str() : "null context"; }

int64_t rp_launch_count(const rp_ctx* ctx) { return ctx ? ctx->launches : 0; }

int rp_set_schedule(rp_ctx* ctx, int32_t policy, int32_t k) {
  if (!ctx) return RP_EINVAL;
  if (policy < RP_SCHED_INDEX || policy > RP_SCHED_SUBREGION) return rp_fail(ctx, RP_EINVAL, "set_schedule: policy");
  if (policy == RP_SCHED_KNN && k != 1 && k != 5 && k != 9 && k != 25)
    return rp_fail(ctx, RP_EINVAL, "set_schedule: k must be 1, 5, 9 or 25");
  ctx->sched_policy = policy;
  ctx->sched_k = policy == RP_SCHED_KNN ? k : 1;
  return RP_OK;
}

int rp_set_work_split(rp_ctx* ctx, int32_t level, int32_t budget) {
  if (!ctx) return RP_EINVAL;
  if (level != 0 && (level < 2 || level > ctx->cfg.max_depth))
    return rp_fail(ctx, RP_EINVAL, "set_work_split: level must be 0 or 2..max_depth");
  if (budget != 0 && (budget < 2 || budget > 64 || (budget & 1)))
    return rp_fail(ctx, RP_EINVAL, "set_work_split: budget must be 0 or even in 2..64");
  ctx->split_level = level;
  ctx->unit_budget = budget ? budget : 64;
  return RP_OK;
}

int rp_set_predictive_partition(rp_ctx* ctx, int32_t mode) {
  RP_ENTER(ctx);
  if (mode != RP_PART_UNIFORM && mode != RP_PART_ADAPTIVE)
    return rp_fail(ctx, RP_EINVAL, "set_predictive_partition: mode must be 0 or 1");
  if (mode == RP_PART_ADAPTIVE && !ctx->leaf_rec) {
    const long long cap =
        std::max(1LL << 22, 4LL * ctx->cfg.nx * ctx->cfg.ny * ctx->cfg.history_depth);
    RP_CUDA(cudaMalloc(&ctx->leaf_rec, (size_t)cap * sizeof(double4)));
    RP_CUDA(cudaMalloc(&ctx->leaf_count_dev, sizeof(unsigned long long)));
    RP_CUDA(cudaMemsetAsync(ctx->leaf_count_dev, 0, sizeof(unsigned long long), ctx->stream));
    ctx->leaf_cap = cap;
  }
  ctx->pred_part = mode;
  ctx->leaf_valid = 0;
  return RP_OK;
}

int rp_predictive_lists_read(rp_ctx* ctx, int64_t* off_host, double* bp_host) {
  if (!ctx) return RP_EINVAL;
  if (ctx->pred_off_host.empty()) return rp_fail(ctx, RP_ESTATE, "predictive_lists: no forecast partition yet");
  if (off_host) std::copy(ctx->pred_off_host.begin(), ctx->pred_off_host.end(), off_host);
  if (bp_host) std::copy(ctx->pred_bp_host.begin(), ctx->pred_bp_host.end(), bp_host);
  return RP_OK;
}

int rp_set_predictive(rp_ctx* ctx, int32_t enable, int32_t knn, int32_t n_clusters,
                      int32_t max_iters) {
  if (!ctx) return RP_EINVAL;
  if (knn != 1 && knn != 5 && knn != 9 && knn != 25)
    return rp_fail(ctx, RP_EINVAL, "set_predictive: k must be 1, 5, 9 or 25");
  if (n_clusters < 0 || max_iters < 1) return rp_fail(ctx, RP_EINVAL, "set_predictive: bad args");
  ctx->pred_on = enable ? 1 : 0;
  ctx->pred_knn = knn;
  ctx->pred_m = n_clusters;
  ctx->pred_iters = max_iters;
  return RP_OK;
}

int rp_predictive_info_read(rp_ctx* ctx, rp_predictive_info* out, int32_t* clusters_host) {
  if (!ctx || !out) return RP_EINVAL;
  *out = ctx->pred_info;
  if (clusters_host) {
    if (!ctx->pred_info.active) return rp_fail(ctx, RP_ESTATE, "predictive_info: no forecast partition yet");
    memcpy(clusters_host, ctx->cluster_host.data(), ctx->cluster_host.size() * sizeof(int32_t));
  }
  return RP_OK;
}

int rp_profile_enable(rp_ctx* ctx, int32_t enable) {
  RP_ENTER(ctx);
  RP_CUDA(cudaStreamSynchronize(ctx->stream));
  for (auto& r : ctx->prof) {
    ctx->ev_pool.push_back(r.a);
    ctx->ev_pool.push_back(r.b);
  }
  ctx->prof.clear();
  for (double& v : ctx->prof_acc) v = 0.0;
  ctx->prof_integrate_launches = 0;
  ctx->prof_on = enable ? 1 : 0;
  return RP_OK;
}

int rp_profile_read(rp_ctx* ctx, rp_profile* out) {
  RP_ENTER(ctx);
  if (!out) return RP_EINVAL;
  RP_CUDA(cudaStreamSynchronize(ctx->stream));
  for (auto& r : ctx->prof) {
    float ms = 0.f;
    RP_CUDA(cudaEventElapsedTime(&ms, r.a, r.b));
    ctx->prof_acc[r.kind] += ms;
    ctx->ev_pool.push_back(r.a);
    ctx->ev_pool.push_back(r.b);
  }
  ctx->prof.clear();
  out->deposit_ms = ctx->prof_acc[PK_DEPOSIT];
  out->append_ms = ctx->prof_acc[PK_APPEND];
  out->clip_ms = ctx->prof_acc[PK_CLIP];
  out->sort_ms = ctx->prof_acc[PK_SORT];
  out->integrate_ms = ctx->prof_acc[PK_INTEGRATE];
  out->reduce_ms = ctx->prof_acc[PK_REDUCE];
  out->fields_ms = ctx->prof_acc[PK_FIELDS];
  out->push_ms = ctx->prof_acc[PK_PUSH];
  out->integrate_launches = ctx->prof_integrate_launches;
  out->units_ms = ctx->prof_acc[PK_UNITS];
  out->step_ms = ctx->prof_acc[PK_STEP];
  return RP_OK;
}

int rp_nccl_unique_id(unsigned char* id_out) {
  if (!id_out) return RP_EINVAL;
  const RpNccl* api = rp_nccl_api(nullptr);
  if (!api) return RP_ENCCL;
  ncclUniqueId id;
  if (api->get_unique_id(&id) != ncclSuccess) return RP_ENCCL;
  memcpy(id_out, &id, RP_NCCL_ID_BYTES);
  return RP_OK;
}

int rp_create(const rp_config* cfg, const rp_dist* dist, rp_ctx** out) {
  if (!out) return RP_EINVAL;
  *out = nullptr;
  if (validate(cfg) != RP_OK) return RP_EINVAL;
  if (dist && (dist->world < 1 || dist->rank < 0 || dist->rank >= dist->world)) return RP_EINVAL;
  int ndev = 0;
  if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev <= cfg->device || cfg->device < 0) {
    cudaGetLastError();
    return RP_ENODEV;
  }
  DeviceGuard guard(cfg->device);  // the caller's device is restored on return
  rp_ctx* ctx = new (std::nothrow) rp_ctx();
  if (!ctx) return RP_ENOMEM;
  ctx->cfg = *cfg;
  auto fail = [&](int rc) {
    free_all(ctx);
    delete ctx;
    return rc;
  };
  if (cudaSetDevice(cfg->device) != cudaSuccess) return fail(RP_ENODEV);
  cudaDeviceGetAttribute(&ctx->sm_count, cudaDevAttrMultiProcessorCount, cfg->device);
  ctx->H = cfg->history_depth + 2;
  ctx->PX = cfg->nx + 2 * RP_PAD;
  ctx->PY = cfg->ny + 2 * RP_PAD;
  ctx->slot_doubles = (size_t)ctx->PX * ctx->PY * 4;
  ctx->fh = new (std::nothrow) rp_frame[ctx->H];
  if (!ctx->fh) return fail(RP_ENOMEM);
  for (int i = 0; i < ctx->H; ++i) ctx->fh[i] = rp_frame{0.0, 0.0, 1.0, 0.0};
  size_t ring_bytes = (size_t)ctx->H * ctx->slot_doubles * sizeof(double);
  if (cudaMalloc(&ctx->ring, ring_bytes) != cudaSuccess) return fail(RP_ENOMEM);
  if (cudaMemset(ctx->ring, 0, ring_bytes) != cudaSuccess) return fail(RP_ECUDA);
  if (cudaMalloc(&ctx->frames_dev, ctx->H * sizeof(rp_frame)) != cudaSuccess) return fail(RP_ENOMEM);
  if (cudaMemcpy(ctx->frames_dev, ctx->fh, ctx->H * sizeof(rp_frame), cudaMemcpyHostToDevice) != cudaSuccess)
    return fail(RP_ECUDA);
  size_t npts = (size_t)cfg->nx * cfg->ny;
  if (cudaMalloc(&ctx->bin_start, (npts + 2) * sizeof(int32_t)) != cudaSuccess) return fail(RP_ENOMEM);
  if (cudaMalloc(&ctx->partial, rp_partial_bytes_impl(ctx)) != cudaSuccess) return fail(RP_ENOMEM);
  int rc = rp_alloc_potential_scratch(ctx);
  if (rc) return fail(rc);
  // analytic amplitudes default to 1
  std::vector<double> ones(ctx->H, 1.0);
  if (cudaMemcpy(ctx->amp_dev, ones.data(), ctx->H * sizeof(double), cudaMemcpyHostToDevice) != cudaSuccess)
    return fail(RP_ECUDA);
  if (dist) {
    ctx->dist_on = 1;
    ctx->rank = dist->rank;
    ctx->world = dist->world;
    const int64_t pb = rp_partial_bytes_impl(ctx);
    ctx->shard_cap = ((int64_t)npts + dist->world - 1) / dist->world;
    if (cudaMalloc(&ctx->partials_all, (size_t)pb * dist->world) != cudaSuccess ||
        cudaMalloc(&ctx->shard_buf, (size_t)ctx->shard_cap * 6 * sizeof(double)) != cudaSuccess ||
        cudaMalloc(&ctx->shards_all, (size_t)ctx->shard_cap * 6 * sizeof(double) * dist->world) != cudaSuccess)
      return fail(RP_ENOMEM);
    if (dist->nccl_comm) {
      ctx->comm = (ncclComm_t)dist->nccl_comm;
    } else {
      std::string e;
      const RpNccl* api = rp_nccl_api(&e);
      if (!api) return fail(RP_ENCCL);
      ncclUniqueId id;
      memcpy(&id, dist->nccl_id, RP_NCCL_ID_BYTES);
      if (api->comm_init_rank(&ctx->comm, dist->world, id, dist->rank) != ncclSuccess) {
        ctx->comm = nullptr;
        return fail(RP_ENCCL);
      }
      ctx->own_comm = 1;
    }
  }
  // the setup copies, memsets and k_iota above ran on the legacy default stream, which a
  // non-blocking caller stream (rp_set_stream) is not ordered after: finish them here
  if (cudaDeviceSynchronize() != cudaSuccess) return fail(RP_ECUDA);
  *out = ctx;
  return RP_OK;
}

void rp_destroy(rp_ctx* ctx) {
  if (!ctx) return;
  DeviceGuard guard(ctx->cfg.device);
  cudaStreamSynchronize(ctx->stream);
  free_all(ctx);
  delete ctx;
}

int rp_set_stream(rp_ctx* ctx, void* stream) {
  if (!ctx) return RP_EINVAL;
  ctx->stream = (cudaStream_t)stream;
  return RP_OK;
}

int rp_history_init(rp_ctx* ctx, int32_t n_pre, const rp_frame* frames_host,
                    const double* grids_dev, int32_t rigid) {
  RP_ENTER(ctx);
  if (ctx->k >= 0) return rp_fail(ctx, RP_ESTATE, "history_init after the first deposit");
  if (n_pre < 1 || n_pre > ctx->cfg.history_depth + 1 || !frames_host)
    return rp_fail(ctx, RP_EINVAL, "history_init: n_pre out of range or no frames");
  if (rigid && grids_dev) return rp_fail(ctx, RP_EINVAL, "history_init: rigid needs grids_dev == NULL");
  if (!rigid && !grids_dev) return rp_fail(ctx, RP_EINVAL, "history_init: grids_dev required");
  const rp_config& c = ctx->cfg;
  for (int i = 0; i < n_pre; ++i) {
    int level = -n_pre + i;
    int s = slot_of(level, ctx->H);
    ctx->fh[s] = frames_host[i];
    if (!rigid) {
      k_pad<<<(c.nx * c.ny + 255) / 256, 256, 0, ctx->stream>>>(
          c.nx, c.ny, ctx->PX, grids_dev + (size_t)i * c.nx * c.ny * 4,
          ctx->ring + (size_t)s * ctx->slot_doubles);
      RP_CHECK_LAUNCH();
    }
  }
  RP_CUDA(cudaMemcpyAsync(ctx->frames_dev, ctx->fh, ctx->H * sizeof(rp_frame), cudaMemcpyHostToDevice,
                          ctx->stream));
  RP_CUDA(cudaStreamSynchronize(ctx->stream));
  ctx->n_pre = n_pre;
  ctx->rigid_pending = rigid ? 1 : 0;
  ctx->prehist_set = 1;
  return RP_OK;
}

int rp_deposit(rp_ctx* ctx, const double* x, const double* y, const double* ux, const double* uy,
               double q, int64_t n, const rp_frame* frame_k, void* partial_dev,
               rp_deposit_info* info) {
  RP_ENTER(ctx);
  return rp_deposit_impl(ctx, x, y, ux, uy, q, n, frame_k, partial_dev, info);
}

int64_t rp_partial_bytes(const rp_ctx* ctx) { return ctx ? rp_partial_bytes_impl(ctx) : 0; }

int rp_history_append(rp_ctx* ctx, const void* partials_dev, int32_t n_parts,
                      const rp_frame* frame_k) {
  RP_ENTER(ctx);
  return rp_append_impl(ctx, partials_dev, n_parts, frame_k);
}

int rp_deposit_step(rp_ctx* ctx, const double* x, const double* y, const double* ux,
                    const double* uy, double q, int64_t n, const rp_frame* frame_k,
                    rp_deposit_info* info) {
  RP_ENTER(ctx);
  return deposit_step(ctx, x, y, ux, uy, q, n, frame_k, info);
}

int rp_compute_potentials(rp_ctx* ctx, double* phi, double* ax, double* ay, double* err,
                          int32_t* nseg, rp_potential_info* info) {
  RP_ENTER(ctx);
  return potentials_full(ctx, phi, ax, ay, err, nseg, info);
}

int64_t rp_shard_capacity(const rp_ctx* ctx, int32_t world) {
  if (!ctx || world < 1) return 0;
  int64_t n = (int64_t)ctx->cfg.nx * ctx->cfg.ny;
  return (n + world - 1) / world;
}

int rp_compute_potentials_shard(rp_ctx* ctx, int32_t rank, int32_t world, double* shard_out,
                                int64_t cap, int64_t* n_out, rp_potential_info* info) {
  RP_ENTER(ctx);
  if (world < 1 || rank < 0 || rank >= world || !shard_out || cap < rp_shard_capacity(ctx, world))
    return rp_fail(ctx, RP_EINVAL, "potentials_shard: bad rank/world/cap");
  if (ctx->pred_on) return rp_fail(ctx, RP_EINVAL, "potentials_shard: Predictive-RP is single-call only");
  return rp_potentials_impl(ctx, RP_SRC_GRID, nullptr, rank, world, nullptr, nullptr, nullptr,
                            nullptr, nullptr, shard_out, cap, n_out, info);
}

int rp_shard_scatter(rp_ctx* ctx, const double* shards, int32_t world, int64_t cap, double* phi,
                     double* ax, double* ay, double* err, int32_t* nseg) {
  RP_ENTER(ctx);
  if (!shards || world < 1 || cap < rp_shard_capacity(ctx, world) || !phi || !ax || !ay)
    return rp_fail(ctx, RP_EINVAL, "shard_scatter: bad args");
  return rp_scatter_impl(ctx, shards, world, cap, phi, ax, ay, err, nseg);
}

int rp_compute_fields(rp_ctx* ctx, const double* phi, const double* ax, const double* ay,
                      const double* a_prev, int32_t n_prev, double* ex, double* ey, double* bz) {
  RP_ENTER(ctx);
  return rp_fields_impl(ctx, phi, ax, ay, a_prev, n_prev, ex, ey, bz);
}

int rp_push_particles(rp_ctx* ctx, double* x, double* y, double* ux, double* uy, int64_t n,
                      double q_over_mc, double bz_ext, const double* ex, const double* ey,
                      const double* bz) {
  RP_ENTER(ctx);
  return rp_push_impl(ctx, x, y, ux, uy, n, q_over_mc, bz_ext, ex, ey, bz);
}

int rp_particle_forces(rp_ctx* ctx, const double* x, const double* y, const double* ux,
                       const double* uy, int64_t n, double bz_ext, const double* ex,
                       const double* ey, const double* bz, double* fx, double* fy) {
  RP_ENTER(ctx);
  return rp_forces_impl(ctx, x, y, ux, uy, n, bz_ext, ex, ey, bz, fx, fy);
}

int rp_kick_external(rp_ctx* ctx, const double* ux, const double* uy, int64_t n,
                     double q_over_mc, double bz_ext, double frac, double* ux_out,
                     double* uy_out) {
  RP_ENTER(ctx);
  return rp_kick_impl(ctx, ux, uy, n, q_over_mc, bz_ext, frac, ux_out, uy_out);
}

int rp_step_host(rp_ctx* ctx, double* xh, double* yh, double* uxh, double* uyh, int64_t n,
                 double q, const rp_frame* frame_k, double q_over_mc, double bz_ext,
                 double* mesh_host, rp_potential_info* info) {
  RP_ENTER(ctx);
  if (n < 0 || (n > 0 && (!xh || !yh || !uxh || !uyh)) || !mesh_host || !frame_k)
    return rp_fail(ctx, RP_EINVAL, "step_host: bad args");
  const size_t npts = (size_t)ctx->cfg.nx * ctx->cfg.ny;
  if (n > ctx->host_cap) {
    cudaFree(ctx->hx_d); cudaFree(ctx->hy_d); cudaFree(ctx->hux_d); cudaFree(ctx->huy_d);
    cudaFree(ctx->cux_d); cudaFree(ctx->cuy_d);
    ctx->hx_d = ctx->hy_d = ctx->hux_d = ctx->huy_d = ctx->cux_d = ctx->cuy_d = nullptr;
    ctx->host_cap = 0;
    RP_CUDA(cudaMalloc(&ctx->hx_d, n * sizeof(double)));
    RP_CUDA(cudaMalloc(&ctx->hy_d, n * sizeof(double)));
    RP_CUDA(cudaMalloc(&ctx->hux_d, n * sizeof(double)));
    RP_CUDA(cudaMalloc(&ctx->huy_d, n * sizeof(double)));
    RP_CUDA(cudaMalloc(&ctx->cux_d, n * sizeof(double)));
    RP_CUDA(cudaMalloc(&ctx->cuy_d, n * sizeof(double)));
    ctx->host_cap = n;
  }
  if (!ctx->mesh_d) RP_CUDA(cudaMalloc(&ctx->mesh_d, 6 * npts * sizeof(double)));
  if (!ctx->aprev_d) RP_CUDA(cudaMalloc(&ctx->aprev_d, 4 * 2 * npts * sizeof(double)));
  cudaStream_t st = ctx->stream;
  size_t nb = (size_t)n * sizeof(double);
  if (n > 0) {
    RP_CUDA(cudaMemcpyAsync(ctx->hx_d, xh, nb, cudaMemcpyHostToDevice, st));
    RP_CUDA(cudaMemcpyAsync(ctx->hy_d, yh, nb, cudaMemcpyHostToDevice, st));
    RP_CUDA(cudaMemcpyAsync(ctx->hux_d, uxh, nb, cudaMemcpyHostToDevice, st));
    RP_CUDA(cudaMemcpyAsync(ctx->huy_d, uyh, nb, cudaMemcpyHostToDevice, st));
  }
  double* m = ctx->mesh_d;
  double *phi = m, *ax = m + npts, *ay = m + 2 * npts, *ex = m + 3 * npts, *ey = m + 4 * npts,
         *bz = m + 5 * npts;
  {
    ProfScope ps(ctx, PK_STEP);  // the device part of the step, between the copies
    // the current of step k with the momenta of t_k (R-27): the leap-frog momenta advanced by
    // half a step in the external field
    int rc = rp_kick_impl(ctx, ctx->hux_d, ctx->huy_d, n, q_over_mc, bz_ext, 0.5, ctx->cux_d,
                          ctx->cuy_d);
    if (rc) return rc;
    rc = deposit_step(ctx, ctx->hx_d, ctx->hy_d, ctx->cux_d, ctx->cuy_d, q, n, frame_k, nullptr);
    if (rc) return rc;
    rc = potentials_full(ctx, phi, ax, ay, nullptr, nullptr, info);
    if (rc) return rc;
    rc = rp_fields_impl(ctx, phi, ax, ay, ctx->aprev_d, ctx->n_prev_A, ex, ey, bz);
    if (rc) return rc;
    // A history for the next step's dA/dt (R-15b): shift, then this step's (A_x, A_y) first
    const size_t pair = 2 * npts * sizeof(double);
    for (int j = 3; j >= 1; --j)
      RP_CUDA(cudaMemcpyAsync(ctx->aprev_d + (size_t)j * 2 * npts,
                              ctx->aprev_d + (size_t)(j - 1) * 2 * npts, pair,
                              cudaMemcpyDeviceToDevice, st));
    RP_CUDA(cudaMemcpyAsync(ctx->aprev_d, ax, pair, cudaMemcpyDeviceToDevice, st));
    ctx->n_prev_A = ctx->n_prev_A < 4 ? ctx->n_prev_A + 1 : 4;
    rc = rp_push_impl(ctx, ctx->hx_d, ctx->hy_d, ctx->hux_d, ctx->huy_d, n, q_over_mc, bz_ext, ex,
                      ey, bz);
    if (rc) return rc;
  }
  RP_CUDA(cudaMemcpyAsync(mesh_host, m, 6 * npts * sizeof(double), cudaMemcpyDeviceToHost, st));
  if (n > 0) {
    RP_CUDA(cudaMemcpyAsync(xh, ctx->hx_d, nb, cudaMemcpyDeviceToHost, st));
    RP_CUDA(cudaMemcpyAsync(yh, ctx->hy_d, nb, cudaMemcpyDeviceToHost, st));
    RP_CUDA(cudaMemcpyAsync(uxh, ctx->hux_d, nb, cudaMemcpyDeviceToHost, st));
    RP_CUDA(cudaMemcpyAsync(uyh, ctx->huy_d, nb, cudaMemcpyDeviceToHost, st));
  }
  RP_CUDA(cudaStreamSynchronize(st));
  return RP_OK;
}

int rp_load_state(rp_ctx* ctx, int32_t k, int32_t n_pre, const rp_frame* frames_host,
                  const double* ring_dev) {
  RP_ENTER(ctx);
  if (k < 0 || n_pre < 0 || n_pre > ctx->cfg.history_depth + 1 || !frames_host || !ring_dev)
    return rp_fail(ctx, RP_EINVAL, "load_state: bad args");
  const rp_config& c = ctx->cfg;
  for (int s = 0; s < ctx->H; ++s) {
    ctx->fh[s] = frames_host[s];
    k_pad<<<(c.nx * c.ny + 255) / 256, 256, 0, ctx->stream>>>(
        c.nx, c.ny, ctx->PX, ring_dev + (size_t)s * c.nx * c.ny * 4,
        ctx->ring + (size_t)s * ctx->slot_doubles);
    RP_CHECK_LAUNCH();
  }
  RP_CUDA(cudaMemcpyAsync(ctx->frames_dev, ctx->fh, ctx->H * sizeof(rp_frame), cudaMemcpyHostToDevice,
                          ctx->stream));
  RP_CUDA(cudaStreamSynchronize(ctx->stream));
  ctx->k = k;
  ctx->n_pre = n_pre;
  ctx->rigid_pending = 0;
  ctx->prehist_set = 1;
  ctx->has_forecast = 0;
  ctx->n_prev_A = 0;
  return RP_OK;
}

int rp_save_state(rp_ctx* ctx, int32_t* k_out, double* ring_dev, rp_frame* frames_host) {
  RP_ENTER(ctx);
  const rp_config& c = ctx->cfg;
  if (k_out) *k_out = ctx->k;
  if (frames_host)
    for (int s = 0; s < ctx->H; ++s) frames_host[s] = ctx->fh[s];
  if (ring_dev) {
    for (int s = 0; s < ctx->H; ++s) {
      k_unpad<<<(c.nx * c.ny + 255) / 256, 256, 0, ctx->stream>>>(
          c.nx, c.ny, ctx->PX, ctx->ring + (size_t)s * ctx->slot_doubles,
          ring_dev + (size_t)s * c.nx * c.ny * 4);
      RP_CHECK_LAUNCH();
    }
  }
  RP_CUDA(cudaStreamSynchronize(ctx->stream));
  return RP_OK;
}

int rp_debug_bins(rp_ctx* ctx, int32_t* bins_dev, int64_t n) {
  RP_ENTER(ctx);
  if (!bins_dev || n != ctx->last_n) return rp_fail(ctx, RP_EINVAL, "debug_bins: n must equal the last deposit's n");
  if (n == 0) return RP_OK;
  k_bins_out<<<(unsigned)((n + 255) / 256), 256, 0, ctx->stream>>>(n, ctx->cfg.nx * ctx->cfg.ny,
                                                                    ctx->keys, bins_dev);
  RP_CHECK_LAUNCH();
  return RP_OK;
}

int rp_debug_point_counts(rp_ctx* ctx, int32_t* nleaf_dev, int32_t* capped_dev, int64_t n) {
  RP_ENTER(ctx);
  const int64_t npts = (int64_t)ctx->cfg.nx * ctx->cfg.ny;
  if (n != npts) return rp_fail(ctx, RP_EINVAL, "debug_point_counts: n must be nx*ny");
  if (!ctx->has_forecast) return rp_fail(ctx, RP_ESTATE, "debug_point_counts: no potentials call yet");
  k_point_counts<<<(unsigned)((n + 255) / 256), 256, 0, ctx->stream>>>(n, ctx->point_cnt, nleaf_dev,
                                                                        capped_dev);
  RP_CHECK_LAUNCH();
  return RP_OK;
}

int rp_debug_item_leaves(rp_ctx* ctx, uint16_t* leaves_dev, int64_t n) {
  RP_ENTER(ctx);
  const int64_t want = (int64_t)ctx->cfg.nx * ctx->cfg.ny * ctx->cfg.history_depth;
  if (!leaves_dev || n != want) return rp_fail(ctx, RP_EINVAL, "debug_item_leaves: n must be nx*ny*history_depth");
  if (!ctx->has_forecast) return rp_fail(ctx, RP_ESTATE, "debug_item_leaves: no potentials call yet");
  RP_CUDA(cudaMemcpyAsync(leaves_dev, ctx->leaves_prev, (size_t)n * sizeof(uint16_t),
                          cudaMemcpyDeviceToDevice, ctx->stream));
  return RP_OK;
}

int rp_debug_clip(rp_ctx* ctx, double* ab_dev, int64_t n) {
  RP_ENTER(ctx);
  const int64_t want = (int64_t)ctx->cfg.nx * ctx->cfg.ny * ctx->cfg.history_depth;
  if (!ab_dev || n != want) return rp_fail(ctx, RP_EINVAL, "debug_clip: n must be nx*ny*history_depth");
  if (!ctx->has_forecast) return rp_fail(ctx, RP_ESTATE, "debug_clip: no potentials call yet");
  RP_CUDA(cudaMemcpyAsync(ab_dev, ctx->clipAB, (size_t)n * sizeof(double2), cudaMemcpyDeviceToDevice,
                          ctx->stream));
  return RP_OK;
}

int rp_debug_potentials_analytic(rp_ctx* ctx, int32_t kind, double x0, double y0, double width,
                                 double q, double bx, double by, const double* amp_host,
                                 double* phi, double* ax, double* ay, double* err, int32_t* nseg,
                                 rp_potential_info* info) {
  RP_ENTER(ctx);
  if ((kind != RP_SRC_GAUSS && kind != RP_SRC_DISK) || !(width > 0))
    return rp_fail(ctx, RP_EINVAL, "debug_potentials_analytic: bad source");
  std::vector<double> h(ctx->H);
  for (int i = 0; i < ctx->H; ++i) h[i] = amp_host ? amp_host[i] : 1.0;
  // stream-ordered upload; the host vector must outlive the copy, hence the sync
  RP_CUDA(cudaMemcpyAsync(ctx->amp_dev, h.data(), ctx->H * sizeof(double), cudaMemcpyHostToDevice,
                          ctx->stream));
  RP_CUDA(cudaStreamSynchronize(ctx->stream));
  double src[6] = {x0, y0, width, q, bx, by};
  int saved = ctx->has_forecast;
  ctx->has_forecast = 0;
  int rc = rp_potentials_impl(ctx, kind, src, 0, 1, phi, ax, ay, err, nseg, nullptr, 0, nullptr, info);
  ctx->has_forecast = saved;
  return rc;
}

}  // extern "C"
