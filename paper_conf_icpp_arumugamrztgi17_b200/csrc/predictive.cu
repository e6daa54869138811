// predictive.cu -- host side of the Predictive-RP variant (rp_set_predictive; DESIGN R-26):
// lines 1-12 of the paper's COMPUTE-POTENTIALS (Algorithm 1), which the paper also
// runs on the CPU.  From the previous call's observed access pattern n_j(p)
// (accepted segments per point and subregion, written by k_reduce):
//   line 3   forecast g(p): kNN regression over the comoving mesh;
//   line 4   COMPUTE-PARTITION: uniform partitioning of S_j into n_j(p) pieces, or
//            adaptive partitioning (R-26b): the item's partition accepted at the
//            previous call (recorded by k_integrate) with each piece cut into
//            max(1, round(n_j / d_j)) equal pieces, a_j and b_j added;
//   line 6   RP-CLUSTERING: k-means of the pattern vectors, m = max(nx, ny);
//   9-12     MERGE-LISTS of the partitions of each cluster.
// The merged lists and the point clusters go to the device; k_integrate (potentials.cu) runs
// lines 13-24: every merged interval cut to an item's support is the root of an adaptive
// dyadic tree.  Deterministic (fixed initial centres, fixed pass order, integer sums), so a
// plain CPU implementation of the same definition reproduces every cluster and breakpoint.
#include <algorithm>
#include <chrono>
#include <thread>
#include <vector>

#include "rp_internal.cuh"

namespace {

// line 3: mean of n_j over the k nearest mesh nodes (index space), rounded half up
inline uint32_t knn_mean(const uint16_t* prev, int nx, int ny, int kmax, int p, int j, int knn) {
  const int ix = p % nx, iy = p / nx;
  const int rad = knn >= 25 ? 2 : (knn >= 5 ? 1 : 0);
  uint32_t sum = 0, cnt = 0;
  for (int dy = -rad; dy <= rad; ++dy)
    for (int dx = -rad; dx <= rad; ++dx) {
      if (knn == 5 && dx != 0 && dy != 0) continue;  // the 4-neighbour cross and the node
      const int x = ix + dx, y = iy + dy;
      if (x < 0 || x >= nx || y < 0 || y >= ny) continue;
      sum += prev[((size_t)y * nx + x) * kmax + j];
      ++cnt;
    }
  return (sum + cnt / 2) / cnt;
}

template <class F>
void parallel_for(int n, F&& f) {
  const int nt = std::max(1, std::min<int>((int)std::thread::hardware_concurrency(), 64));
  if (nt == 1 || n < 256) {
    for (int i = 0; i < n; ++i) f(i);
    return;
  }
  std::vector<std::thread> th;
  const int chunk = (n + nt - 1) / nt;
  for (int t = 0; t < nt; ++t)
    th.emplace_back([&, t] {
      const int lo = t * chunk, hi = std::min(n, lo + chunk);
      for (int i = lo; i < hi; ++i) f(i);
    });
  for (auto& x : th) x.join();
}

// line 6: Lloyd k-means from the centres a(floor(c * n / m)); the nearest centre by squared
// distance summed over j in ascending order (first minimum wins); centres = integer member
// sums / member counts (empty clusters keep theirs); stop when nothing moves or after
// max_iters assignment passes.  Returns the passes made.
int kmeans(const std::vector<uint16_t>& a, int n, int d, int m, int max_iters,
           std::vector<int32_t>& lab) {
  std::vector<double> mu((size_t)m * d);
  for (int c = 0; c < m; ++c) {
    const size_t src = (size_t)((int64_t)c * n / m) * d;
    for (int j = 0; j < d; ++j) mu[(size_t)c * d + j] = (double)a[src + j];
  }
  lab.assign(n, -1);
  std::vector<int64_t> sum((size_t)m * d), cnt(m);
  std::vector<uint8_t> moved(n);
  int passes = 0;
  for (;;) {
    ++passes;
    parallel_for(n, [&](int p) {
      const uint16_t* x = a.data() + (size_t)p * d;
      int best = 0;
      double bd = 0.0;
      for (int c = 0; c < m; ++c) {
        const double* y = mu.data() + (size_t)c * d;
        double s = 0.0;
        for (int j = 0; j < d; ++j) {
          const double e = (double)x[j] - y[j];
          s += e * e;
        }
        if (c == 0 || s < bd) {
          bd = s;
          best = c;
        }
      }
      moved[p] = lab[p] != best;
      lab[p] = best;
    });
    bool any = false;
    for (int p = 0; p < n; ++p) any |= moved[p] != 0;
    if (!any || passes >= max_iters) break;
    std::fill(sum.begin(), sum.end(), 0);
    std::fill(cnt.begin(), cnt.end(), 0);
    for (int p = 0; p < n; ++p) {
      const int c = lab[p];
      ++cnt[c];
      for (int j = 0; j < d; ++j) sum[(size_t)c * d + j] += a[(size_t)p * d + j];
    }
    for (int c = 0; c < m; ++c)
      if (cnt[c])
        for (int j = 0; j < d; ++j) mu[(size_t)c * d + j] = (double)sum[(size_t)c * d + j] / (double)cnt[c];
  }
  return passes;
}

}  // namespace

int rp_predictive_setup(rp_ctx* ctx, int kap) {
  const auto t0 = std::chrono::steady_clock::now();
  const rp_config& cf = ctx->cfg;
  const int nx = cf.nx, ny = cf.ny, n = nx * ny, d = cf.history_depth;
  // observed pattern of the previous call (k_reduce); the download orders after it
  std::vector<uint16_t> prev((size_t)n * d), pat((size_t)n * d, 0);
  RP_CUDA(cudaMemcpyAsync(prev.data(), ctx->leaves_prev, prev.size() * sizeof(uint16_t),
                          cudaMemcpyDeviceToHost, ctx->stream));
  RP_CUDA(cudaStreamSynchronize(ctx->stream));
  parallel_for(n, [&](int p) {
    for (int j = 0; j < kap; ++j)
      pat[(size_t)p * d + j] = (uint16_t)std::min<uint32_t>(
          knn_mean(prev.data(), nx, ny, d, p, j, ctx->pred_knn), 0xFFFF);
  });
  int m = ctx->pred_m > 0 ? ctx->pred_m : std::max(nx, ny);
  m = std::min(m, n);
  std::vector<int32_t>& lab = ctx->cluster_host;
  const int passes = kmeans(pat, n, d, m, ctx->pred_iters, lab);
  // line 4 by adaptive partitioning: the previous call's accepted partition of every
  // item, from the leaf records (a, b, item): per item the left ends in r' order, then the
  // last right end (the leaves tile the item's support)
  int adaptive = ctx->pred_part == RP_PART_ADAPTIVE ? 1 : 0;
  std::vector<int64_t> poff;
  std::vector<int32_t> plen;
  std::vector<double> parts;
  if (adaptive) {
    unsigned long long cnt = 0;
    if (ctx->leaf_valid) {
      RP_CUDA(cudaMemcpyAsync(&cnt, ctx->leaf_count_dev, sizeof(cnt), cudaMemcpyDeviceToHost,
                              ctx->stream));
      RP_CUDA(cudaStreamSynchronize(ctx->stream));
    }
    if (!ctx->leaf_valid || cnt > (unsigned long long)ctx->leaf_cap) {
      adaptive = -1;  // no (complete) earlier partition: uniform partitioning this call
      if (ctx->leaf_valid) {  // grow for the next call
        cudaFree(ctx->leaf_rec);
        ctx->leaf_rec = nullptr;
        const long long cap = (long long)(2 * cnt);
        RP_CUDA(cudaMalloc(&ctx->leaf_rec, (size_t)cap * sizeof(double4)));
        ctx->leaf_cap = cap;
      }
    } else {
      std::vector<double4> rec((size_t)cnt);
      if (cnt) {
        RP_CUDA(cudaMemcpyAsync(rec.data(), ctx->leaf_rec, cnt * sizeof(double4),
                                cudaMemcpyDeviceToHost, ctx->stream));
        RP_CUDA(cudaStreamSynchronize(ctx->stream));
      }
      if (2 * cnt > (unsigned long long)ctx->leaf_cap) {  // keep room for this call's leaves
        cudaFree(ctx->leaf_rec);
        ctx->leaf_rec = nullptr;
        const long long cap = (long long)(4 * cnt);
        RP_CUDA(cudaMalloc(&ctx->leaf_rec, (size_t)cap * sizeof(double4)));
        ctx->leaf_cap = cap;
      }
      std::sort(rec.begin(), rec.end(), [](const double4& x, const double4& y) {
        return x.z < y.z || (x.z == y.z && x.x < y.x);
      });
      poff.assign((size_t)n * d, 0);
      plen.assign((size_t)n * d, 0);
      parts.reserve(rec.size() + rec.size() / 4 + 1);
      for (size_t i = 0; i < rec.size();) {
        size_t e = i;
        while (e < rec.size() && rec[e].z == rec[i].z) ++e;
        const size_t item = (size_t)rec[i].z;
        poff[item] = (int64_t)parts.size();
        for (size_t t = i; t < e; ++t) parts.push_back(rec[t].x);
        parts.push_back(rec[e - 1].y);
        plen[item] = (int32_t)(e - i + 1);
        i = e;
      }
    }
  }
  // lines 4, 9-12: per (cluster, j) the sorted union of the members' partitions of S_j
  std::vector<std::vector<int>> mem(adaptive == 1 ? m : 0);
  if (adaptive == 1)
    for (int p = 0; p < n; ++p) mem[lab[p]].push_back(p);
  std::vector<std::vector<int>> ns((size_t)m * d);
  for (int p = 0; p < n; ++p)
    for (int j = 0; j < kap; ++j) {
      const int v = pat[(size_t)p * d + j];
      if (v > 0) ns[(size_t)lab[p] * d + j].push_back(v);
    }
  const double cdt = cf.c * cf.dt;
  std::vector<int64_t> off((size_t)m * d + 1);
  std::vector<std::vector<double>> lists((size_t)m * d);
  parallel_for(m * d, [&](int i) {
    if (adaptive == 1) {
      const int c = i / d, j = i % d;
      const double aj = (double)j * cdt, bj = (double)(j + 1) * cdt;
      std::vector<double>& L = lists[i];
      for (int p : mem[c]) {
        const int q0 = pat[(size_t)p * d + j];
        if (q0 == 0) continue;
        const size_t it = (size_t)p * d + j;
        if (plen[it] >= 2) {  // each earlier piece into max(1, round(n / d)) pieces
          const double* x = parts.data() + poff[it];
          const int dd = plen[it] - 1;
          const int q = std::max(1, (2 * q0 + dd) / (2 * dd));
          L.push_back(aj);
          L.push_back(bj);
          for (int k = 1; k <= dd; ++k)
            for (int t = 0; t < q; ++t) L.push_back(x[k - 1] + (x[k] - x[k - 1]) * ((double)t / (double)q));
          L.push_back(x[dd]);
        } else {  // no earlier partition of S_j: uniform
          for (int t = 0; t <= q0; ++t) L.push_back(t == q0 ? bj : aj + (bj - aj) * ((double)t / (double)q0));
        }
      }
      std::sort(L.begin(), L.end());
      L.erase(std::unique(L.begin(), L.end()), L.end());
      return;
    }
    std::vector<int>& v = ns[i];
    std::sort(v.begin(), v.end());
    v.erase(std::unique(v.begin(), v.end()), v.end());
    if (v.empty()) return;
    const int j = i % d;
    const double a = (double)j * cdt, b = (double)(j + 1) * cdt;
    std::vector<double>& L = lists[i];
    for (int q : v)
      for (int t = 0; t <= q; ++t) L.push_back(t == q ? b : a + (b - a) * ((double)t / (double)q));
    std::sort(L.begin(), L.end());
    L.erase(std::unique(L.begin(), L.end()), L.end());
  });
  int64_t tot = 0;
  for (size_t i = 0; i < lists.size(); ++i) {
    off[i] = tot;
    tot += (int64_t)lists[i].size();
  }
  off[lists.size()] = tot;
  std::vector<double> bp((size_t)std::max<int64_t>(tot, 1));
  for (size_t i = 0; i < lists.size(); ++i)
    std::copy(lists[i].begin(), lists[i].end(), bp.begin() + off[i]);
  ctx->pred_off_host = off;  // kept for rp_predictive_lists_read (parity with the oracle)
  ctx->pred_bp_host.assign(bp.begin(), bp.begin() + tot);
  // upload on the context's stream (a non-blocking stream is not ordered after copies on the
  // legacy default stream), then wait, so the host vectors may go out of scope
  if ((int64_t)off.size() > ctx->off_cap) {
    if (ctx->bp_off_dev) cudaFree(ctx->bp_off_dev);
    ctx->bp_off_dev = nullptr;
    RP_CUDA(cudaMalloc(&ctx->bp_off_dev, off.size() * sizeof(int64_t)));
    ctx->off_cap = (int64_t)off.size();
  }
  if ((int64_t)bp.size() > ctx->bp_cap) {
    if (ctx->bp_dev) cudaFree(ctx->bp_dev);
    ctx->bp_dev = nullptr;
    RP_CUDA(cudaMalloc(&ctx->bp_dev, bp.size() * sizeof(double)));
    ctx->bp_cap = (int64_t)bp.size();
  }
  RP_CUDA(cudaMemcpyAsync(ctx->bp_off_dev, off.data(), off.size() * sizeof(int64_t),
                          cudaMemcpyHostToDevice, ctx->stream));
  RP_CUDA(cudaMemcpyAsync(ctx->bp_dev, bp.data(), bp.size() * sizeof(double),
                          cudaMemcpyHostToDevice, ctx->stream));
  RP_CUDA(cudaMemcpyAsync(ctx->cluster_dev, lab.data(), n * sizeof(int32_t),
                          cudaMemcpyHostToDevice, ctx->stream));
  RP_CUDA(cudaStreamSynchronize(ctx->stream));
  ctx->pred_info.active = 1;
  ctx->pred_info.partition = adaptive == 1 ? RP_PART_ADAPTIVE : adaptive == -1 ? -1 : RP_PART_UNIFORM;
  ctx->pred_info.clusters = m;
  ctx->pred_info.kmeans_passes = passes;
  ctx->pred_info.breakpoints = tot;
  ctx->pred_info.host_ms =
      std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
  return RP_OK;
}
