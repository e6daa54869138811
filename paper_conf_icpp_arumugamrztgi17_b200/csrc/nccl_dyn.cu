// nccl_dyn.cu -- NCCL for librp's multi-GPU exchange (all-gather of the per-rank
// partial moment grids after deposition and of the potential shards after integration).
//
// NCCL is resolved at run time (dlopen) the first time a context is created with an rp_dist,
// so librp loads -- and its single-GPU path runs -- on machines without NCCL, and a process
// that already holds a libnccl.so.2 (e.g. the one torch links) reuses that copy instead of
// mapping a second NCCL next to it.  Only the types come from nccl.h.
#include <dlfcn.h>
#include <nccl.h>

#include <mutex>
#include <string>

#include "rp_internal.cuh"

namespace {

std::mutex g_mu;
RpNccl g_api;
bool g_tried = false;
std::string g_err;

template <typename F>
bool sym(void* h, const char* name, F& out) {
  out = reinterpret_cast<F>(dlsym(h, name));
  return out != nullptr;
}

}  // namespace

const RpNccl* rp_nccl_api(std::string* err) {
  std::lock_guard<std::mutex> lk(g_mu);
  if (!g_tried) {
    g_tried = true;
    // an NCCL already mapped into the process first (same soname), then the loader's search
    void* h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_NOLOAD);
    if (!h) h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_LOCAL);
    if (!h) h = dlopen("libnccl.so", RTLD_NOW | RTLD_LOCAL);
    if (!h) {
      const char* e = dlerror();
      g_err = std::string("cannot load libnccl.so.2: ") + (e ? e : "?");
    } else {
      RpNccl a{};
      a.handle = h;
      bool ok = sym(h, "ncclGetUniqueId", a.get_unique_id) &&
                sym(h, "ncclCommInitRank", a.comm_init_rank) &&
                sym(h, "ncclCommDestroy", a.comm_destroy) &&
                sym(h, "ncclAllGather", a.all_gather) &&
                sym(h, "ncclGetErrorString", a.error_string) &&
                sym(h, "ncclGetVersion", a.get_version);
      if (ok) {
        g_api = a;
      } else {
        g_err = "libnccl.so.2 lacks a required symbol";
      }
    }
  }
  if (!g_api.handle) {
    if (err) *err = g_err;
    return nullptr;
  }
  return &g_api;
}

static_assert(sizeof(ncclUniqueId) == RP_NCCL_ID_BYTES, "ncclUniqueId size");
static_assert(ncclUint8 == 1, "ncclDataType_t");
