// deposit.cu -- step 1 of the paper's loop: particle deposition onto the grid of
// moments D_k, and the history append.  Atomics-free sorted-bin scatter:
//   k_bin        particle -> nearest node (bit-exact, no FMA; R-13), TSC offsets, beta
//   CUB sort     stable radix sort of (bin, particle id)
//   k_bin_start  per-bin start offsets (binary search in the sorted keys)
//   k_gather     particle records into sorted order (coalesced reads below)
//   k_node_sum   one warp per node: sum over its 9 neighbour bins -> exact partial M_k
//   k_append     D_k = exact sum of the per-rank partials -> ring slot k mod H
// Partial sums are exact: every particle contribution is rounded once to a 128-bit fixed-point
// number (quantum 2^-shift, shift from |q|/(hx hy) so 2^40 particles cannot overflow) and the
// integer sums are order-independent, so D_k is bit-identical however the particles are split
// over ranks, lanes or warps.  The one rounding to FP64 happens in k_append.
#include <algorithm>

#include <cub/device/device_radix_sort.cuh>

#include "rp_internal.cuh"

namespace {

__global__ void k_bin(int64_t n, const double* __restrict__ x, const double* __restrict__ y,
                      const double* __restrict__ ux, const double* __restrict__ uy,
                      rp_frame F, double hx, double hy, int nx, int ny,
                      int32_t* __restrict__ key, int32_t* __restrict__ perm,
                      double4* __restrict__ rec) {
  int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (i >= n) return;
  // local coordinates and nearest node: IEEE round-to-nearest, no contraction (R-13)
  double dx = __dsub_rn(x[i], F.ox), dy = __dsub_rn(y[i], F.oy);
  double u = __dadd_rn(__dmul_rn(F.cos_psi, dx), __dmul_rn(F.sin_psi, dy));
  double v = __dsub_rn(__dmul_rn(F.cos_psi, dy), __dmul_rn(F.sin_psi, dx));
  double tx = __ddiv_rn(u, hx), ty = __ddiv_rn(v, hy);
  double fx = floor(__dadd_rn(tx, 0.5)), fy = floor(__dadd_rn(ty, 0.5));
  bool ok = fx >= 1.0 && fx <= (double)(nx - 2) && fy >= 1.0 && fy <= (double)(ny - 2);
  double a = ux[i], b = uy[i];
  double g = sqrt(1.0 + a * a + b * b);
  key[i] = ok ? (int32_t)fy * nx + (int32_t)fx : nx * ny;
  perm[i] = (int32_t)i;
  rec[i] = make_double4(__dsub_rn(tx, fx), __dsub_rn(ty, fy), a / g, b / g);
}

__global__ void k_bin_start(const int32_t* __restrict__ keys, int64_t n, int nbins,
                            int32_t* __restrict__ start) {
  int b = blockIdx.x * blockDim.x + threadIdx.x;
  if (b > nbins) return;
  int64_t lo = 0, hi = n;  // first index with keys[idx] >= b
  while (lo < hi) {
    int64_t m = (lo + hi) >> 1;
    if (keys[m] < b) lo = m + 1; else hi = m;
  }
  start[b] = (int32_t)lo;
}

__global__ void k_gather(int64_t n, const int32_t* __restrict__ perm,
                         const double4* __restrict__ rec, double4* __restrict__ out) {
  int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (i < n) out[i] = rec[perm[i]];
}

__device__ __forceinline__ void tsc(double d, double& wm, double& w0, double& wp) {
  double a = 0.5 - d, b = 0.5 + d;
  wm = 0.5 * (a * a);
  w0 = 0.75 - d * d;
  wp = 0.5 * (b * b);
}

__device__ __forceinline__ __int128 to_fixed(double v, int shift) {
  return (__int128)rint(ldexp(v, shift));
}

__device__ __forceinline__ __int128 shfl_xor_i128(__int128 v, int o) {
  unsigned long long lo = (unsigned long long)v, hi = (unsigned long long)(v >> 64);
  lo = __shfl_xor_sync(0xffffffffu, lo, o);
  hi = __shfl_xor_sync(0xffffffffu, hi, o);
  return (__int128)(((unsigned __int128)hi << 64) | lo);
}

// One warp per grid node.  Node (ix, iy) receives from the particles of bin
// (ix - oa, iy - ob), oa, ob in {-1, 0, 1}, the weight w_oa(dx) w_ob(dy) (TSC).
// out: [nx*ny][3] 128-bit fixed-point sums (rho, rho*bx, rho*by) x 2^shift.
__global__ void k_node_sum(int nx, int ny, const int32_t* __restrict__ start,
                           const double4* __restrict__ rec, double scale, int shift,
                           __int128* __restrict__ out) {
  int warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  int lane = threadIdx.x & 31;
  if (warp >= nx * ny) return;
  int ix = warp % nx, iy = warp / nx;
  __int128 s0 = 0, s1 = 0, s2 = 0;
  for (int ob = -1; ob <= 1; ++ob) {
    int by = iy - ob;
    if (by < 1 || by > ny - 2) continue;
    for (int oa = -1; oa <= 1; ++oa) {
      int bx = ix - oa;
      if (bx < 1 || bx > nx - 2) continue;
      int b = by * nx + bx;
      int p0 = start[b], p1 = start[b + 1];
      for (int p = p0 + lane; p < p1; p += 32) {
        double4 r = rec[p];
        double wm, w0, wp, vm, v0, vp;
        tsc(r.x, wm, w0, wp);
        tsc(r.y, vm, v0, vp);
        double wx = oa < 0 ? wm : (oa == 0 ? w0 : wp);
        double wy = ob < 0 ? vm : (ob == 0 ? v0 : vp);
        double w = scale * (wx * wy);  // q w_a w_b / (hx hy), one rounding per particle
        s0 += to_fixed(w, shift);
        s1 += to_fixed(w * r.z, shift);
        s2 += to_fixed(w * r.w, shift);
      }
    }
  }
  for (int o = 16; o > 0; o >>= 1) {
    s0 += shfl_xor_i128(s0, o);
    s1 += shfl_xor_i128(s1, o);
    s2 += shfl_xor_i128(s2, o);
  }
  if (lane == 0) {
    __int128* m = out + 3 * (size_t)warp;
    m[0] = s0;
    m[1] = s1;
    m[2] = s2;
  }
}

// ring slot (padded) <- exact sum of n_parts partial buffers (header + [npts][3] int128)
__global__ void k_append(int nx, int ny, int PX, const unsigned char* __restrict__ parts,
                         size_t part_bytes, int n_parts, double* __restrict__ slot) {
  int id = blockIdx.x * blockDim.x + threadIdx.x;
  if (id >= nx * ny) return;
  int ix = id % nx, iy = id / nx;
  __int128 a = 0, b = 0, c = 0;
  // common quantum: the coarsest of the parts (smallest shift), so no part is shifted left
  // (which could overflow); equal shifts -- the same q on every rank -- keep the sum exact,
  // a finer part is rounded to the common quantum (half up), in part order: deterministic
  int shift = 1 << 30;
  for (int i = 0; i < n_parts; ++i)
    shift = min(shift, (int)reinterpret_cast<const long long*>(parts + i * part_bytes)[0]);
  for (int i = 0; i < n_parts; ++i) {
    const unsigned char* base = parts + i * part_bytes;
    const int d = (int)reinterpret_cast<const long long*>(base)[0] - shift;  // >= 0
    const __int128* m = reinterpret_cast<const __int128*>(base + 16) + 3 * (size_t)id;
    if (d == 0) {
      a += m[0]; b += m[1]; c += m[2];
    } else if (d < 126) {  // |part| < 2^126: a shift by >= 126 rounds it to 0
      const __int128 half = (__int128)1 << (d - 1);
      a += (m[0] + half) >> d;
      b += (m[1] + half) >> d;
      c += (m[2] + half) >> d;
    }
  }
  double* dst = slot + 4 * ((size_t)(iy + RP_PAD) * PX + (ix + RP_PAD));
  dst[0] = ldexp((double)a, -shift);
  dst[1] = ldexp((double)b, -shift);
  dst[2] = ldexp((double)c, -shift);
  dst[3] = 0.0;
}

// Rigid steady-state pre-history (R-23): level l gets the step-0 moments with the current
// rotated from frame 0 to frame l, J_l = R(psi_l - psi_0) J_0, so that every level holds the
// same comoving bunch (same local (J.t, J.n)).  cos/sin of the difference angle from the
// frames' (cos, sin) pairs; explicit _rn operations (no FMA contraction) so the copy is a
// fixed function of the inputs.  Static frames give cd = 1, sd = 0: an exact copy.
__global__ void k_rigid_copy(const double* __restrict__ src, double* __restrict__ dst,
                             size_t nodes, rp_frame f0, rp_frame fl) {
  const double cd = __dadd_rn(__dmul_rn(fl.cos_psi, f0.cos_psi), __dmul_rn(fl.sin_psi, f0.sin_psi));
  const double sd = __dsub_rn(__dmul_rn(fl.sin_psi, f0.cos_psi), __dmul_rn(fl.cos_psi, f0.sin_psi));
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < nodes;
       i += (size_t)gridDim.x * blockDim.x) {
    const double4 m = reinterpret_cast<const double4*>(src)[i];
    double4 o;
    o.x = m.x;
    o.y = __dsub_rn(__dmul_rn(cd, m.y), __dmul_rn(sd, m.z));
    o.z = __dadd_rn(__dmul_rn(sd, m.y), __dmul_rn(cd, m.z));
    o.w = m.w;
    reinterpret_cast<double4*>(dst)[i] = o;
  }
}

// frame upload as a kernel parameter: stream-ordered and capturable (no host pointer kept)
__global__ void k_set_frame(rp_frame* dst, rp_frame f) { *dst = f; }

__global__ void k_set_header(long long* hdr, long long shift) {
  hdr[0] = shift;
  hdr[1] = 0;
}

int grow_deposit(rp_ctx* ctx, int64_t n) {
  if (n <= ctx->dep_cap) return RP_OK;
  int64_t cap = n + n / 8 + 1024;
  cudaFree(ctx->keys); cudaFree(ctx->keys_sorted); cudaFree(ctx->perm);
  cudaFree(ctx->perm_sorted); cudaFree(ctx->rec); cudaFree(ctx->rec_sorted);
  ctx->keys = ctx->keys_sorted = ctx->perm = ctx->perm_sorted = nullptr;
  ctx->rec = ctx->rec_sorted = nullptr;
  ctx->dep_cap = 0;
  RP_CUDA(cudaMalloc(&ctx->keys, cap * sizeof(int32_t)));
  RP_CUDA(cudaMalloc(&ctx->keys_sorted, cap * sizeof(int32_t)));
  RP_CUDA(cudaMalloc(&ctx->perm, cap * sizeof(int32_t)));
  RP_CUDA(cudaMalloc(&ctx->perm_sorted, cap * sizeof(int32_t)));
  RP_CUDA(cudaMalloc(&ctx->rec, cap * sizeof(double4)));
  RP_CUDA(cudaMalloc(&ctx->rec_sorted, cap * sizeof(double4)));
  ctx->dep_cap = cap;
  return RP_OK;
}

}  // namespace

int rp_ensure_cub_tmp(rp_ctx* ctx, size_t bytes) {
  if (bytes <= ctx->cub_tmp_bytes) return RP_OK;
  cudaFree(ctx->cub_tmp);
  ctx->cub_tmp = nullptr;
  ctx->cub_tmp_bytes = 0;
  size_t b = bytes + bytes / 4 + 4096;
  RP_CUDA(cudaMalloc(&ctx->cub_tmp, b));
  ctx->cub_tmp_bytes = b;
  return RP_OK;
}

int64_t rp_partial_bytes_impl(const rp_ctx* ctx) {
  return 16 + (int64_t)ctx->cfg.nx * ctx->cfg.ny * 3 * 16;
}

// quantum of the exact partial sums: |sum| <= |q| N / (hx hy) < 2^126 for N <= 2^40
static int fixed_shift(double q, double hx, double hy) {
  double a = fabs(q) / (hx * hy);
  if (!(a > 0.0) || !isfinite(a)) return 64;
  return 126 - 40 - 1 - (int)ceil(log2(a));
}

int rp_deposit_impl(rp_ctx* ctx, const double* x, const double* y, const double* ux,
                    const double* uy, double q, int64_t n, const rp_frame* fk,
                    void* partial, rp_deposit_info* info) {
  const rp_config& c = ctx->cfg;
  if (n < 0 || n > 0x7fffffffLL || !fk || !partial) return rp_fail(ctx, RP_EINVAL, "deposit: bad args");
  if (n > 0 && (!x || !y || !ux || !uy)) return rp_fail(ctx, RP_EINVAL, "deposit: null particle array");
  int rc = grow_deposit(ctx, n > 0 ? n : 1);
  if (rc) return rc;
  const int nbins = c.nx * c.ny;  // + 1 "lost" bin with key nbins
  cudaStream_t st = ctx->stream;
  ctx->last_n = n;
  ProfScope ps(ctx, PK_DEPOSIT);
  if (n > 0) {
    int T = 256;
    k_bin<<<(unsigned)((n + T - 1) / T), T, 0, st>>>(n, x, y, ux, uy, *fk, c.hx, c.hy, c.nx,
                                                      c.ny, ctx->keys, ctx->perm, ctx->rec);
    RP_CHECK_LAUNCH();
    int end_bit = 1;
    while ((1LL << end_bit) <= nbins) ++end_bit;
    size_t tmp = 0;
    RP_CUDA(cub::DeviceRadixSort::SortPairs(nullptr, tmp, ctx->keys, ctx->keys_sorted, ctx->perm,
                                            ctx->perm_sorted, (int)n, 0, end_bit, st));
    rc = rp_ensure_cub_tmp(ctx, tmp);
    if (rc) return rc;
    tmp = ctx->cub_tmp_bytes;
    RP_CUDA(cub::DeviceRadixSort::SortPairs(ctx->cub_tmp, tmp, ctx->keys, ctx->keys_sorted,
                                            ctx->perm, ctx->perm_sorted, (int)n, 0, end_bit, st));
    k_bin_start<<<(nbins + 1 + 255) / 256, 256, 0, st>>>(ctx->keys_sorted, n, nbins, ctx->bin_start);
    RP_CHECK_LAUNCH();
    k_gather<<<(unsigned)((n + T - 1) / T), T, 0, st>>>(n, ctx->perm_sorted, ctx->rec, ctx->rec_sorted);
    RP_CHECK_LAUNCH();
  } else {
    RP_CUDA(cudaMemsetAsync(ctx->bin_start, 0, (nbins + 1) * sizeof(int32_t), st));
  }
  double scale = q / (c.hx * c.hy);
  const int shift = fixed_shift(q, c.hx, c.hy);
  k_set_header<<<1, 1, 0, st>>>(reinterpret_cast<long long*>(partial), shift);
  RP_CHECK_LAUNCH();
  int warps_per_block = 8;
  k_node_sum<<<(nbins + warps_per_block - 1) / warps_per_block, 32 * warps_per_block, 0, st>>>(
      c.nx, c.ny, ctx->bin_start, ctx->rec_sorted, scale, shift,
      reinterpret_cast<__int128*>(reinterpret_cast<unsigned char*>(partial) + 16));
  RP_CHECK_LAUNCH();
  if (info) {
    int32_t kept = 0;
    RP_CUDA(cudaMemcpyAsync(&kept, ctx->bin_start + nbins, sizeof(int32_t), cudaMemcpyDeviceToHost, st));
    RP_CUDA(cudaStreamSynchronize(st));
    if (n == 0) kept = 0;
    info->n_lost = n - kept;
    info->q_lost = q * (double)(n - kept);
    info->q_total = q * (double)n;
  }
  return RP_OK;
}

int rp_append_impl(rp_ctx* ctx, const void* parts, int32_t n_parts, const rp_frame* fk) {
  const rp_config& c = ctx->cfg;
  if (!parts || n_parts < 1 || !fk) return rp_fail(ctx, RP_EINVAL, "append: bad args");
  cudaStream_t st = ctx->stream;
  int knew = ctx->k + 1;
  int s = slot_of(knew, ctx->H);
  double* slot = ctx->ring + (size_t)s * ctx->slot_doubles;
  int npts = c.nx * c.ny;
  ProfScope ps(ctx, PK_APPEND);
  k_append<<<(npts + 255) / 256, 256, 0, st>>>(c.nx, c.ny, ctx->PX,
                                                reinterpret_cast<const unsigned char*>(parts),
                                                (size_t)rp_partial_bytes_impl(ctx), n_parts, slot);
  RP_CHECK_LAUNCH();
  ctx->fh[s] = *fk;
  k_set_frame<<<1, 1, 0, st>>>(ctx->frames_dev + s, *fk);
  RP_CHECK_LAUNCH();
  if (knew == 0 && ctx->rigid_pending) {
    const size_t nodes = ctx->slot_doubles / 4;
    for (int l = -ctx->n_pre; l < 0; ++l) {
      const int sl = slot_of(l, ctx->H);
      double* d = ctx->ring + (size_t)sl * ctx->slot_doubles;
      k_rigid_copy<<<(unsigned)std::min<size_t>((nodes + 255) / 256, 4 * 148), 256, 0, st>>>(
          slot, d, nodes, *fk, ctx->fh[sl]);
      RP_CHECK_LAUNCH();
    }
    ctx->rigid_pending = 0;
  }
  ctx->k = knew;
  return RP_OK;
}
