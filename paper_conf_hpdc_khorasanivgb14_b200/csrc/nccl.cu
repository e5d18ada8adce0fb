// nccl.cu — the multi-GPU exchange of row (e) over NCCL (NVLink 5 / NVSwitch).
//
// libnccl.so.2 is opened at run time (dlopen), so single-GPU use has no NCCL
// dependency; torch ships the library and has normally loaded it already.
// Per iteration every rank broadcasts, in one NCCL group, its slice of the
// write-back values (gathered[], 4 B per owned vertex) and of active[] (1 B
// per owned shard); after convergence the VertexValues slices are broadcast
// once so that cusha_get_values returns |V| values on every rank.
#include <dlfcn.h>
#include <nccl.h>

#include <algorithm>
#include <cstring>
#include <string>

#include "graph.hpp"

namespace cusha {

namespace {
struct NcclApi {
  bool ok = false;
  std::string why;
  decltype(&ncclGetUniqueId) getUniqueId = nullptr;
  decltype(&ncclCommInitRank) commInitRank = nullptr;
  decltype(&ncclCommDestroy) commDestroy = nullptr;
  decltype(&ncclBroadcast) broadcast = nullptr;
  decltype(&ncclGroupStart) groupStart = nullptr;
  decltype(&ncclGroupEnd) groupEnd = nullptr;
  decltype(&ncclGetErrorString) errorString = nullptr;
};

const NcclApi& api() {
  static NcclApi a = [] {
    NcclApi x;
    void* h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
    if (!h) h = dlopen("libnccl.so", RTLD_NOW | RTLD_GLOBAL);
    if (!h) {
      x.why = std::string("dlopen(libnccl.so.2) failed: ") + dlerror();
      return x;
    }
    x.getUniqueId = reinterpret_cast<decltype(x.getUniqueId)>(dlsym(h, "ncclGetUniqueId"));
    x.commInitRank = reinterpret_cast<decltype(x.commInitRank)>(dlsym(h, "ncclCommInitRank"));
    x.commDestroy = reinterpret_cast<decltype(x.commDestroy)>(dlsym(h, "ncclCommDestroy"));
    x.broadcast = reinterpret_cast<decltype(x.broadcast)>(dlsym(h, "ncclBroadcast"));
    x.groupStart = reinterpret_cast<decltype(x.groupStart)>(dlsym(h, "ncclGroupStart"));
    x.groupEnd = reinterpret_cast<decltype(x.groupEnd)>(dlsym(h, "ncclGroupEnd"));
    x.errorString = reinterpret_cast<decltype(x.errorString)>(dlsym(h, "ncclGetErrorString"));
    x.ok = x.getUniqueId && x.commInitRank && x.commDestroy && x.broadcast && x.groupStart && x.groupEnd &&
           x.errorString;
    if (!x.ok) x.why = "libnccl.so.2 lacks a required symbol";
    return x;
  }();
  return a;
}

#define NC(call)                                                                           \
  do {                                                                                     \
    ncclResult_t r_ = (call);                                                              \
    if (r_ != ncclSuccess) {                                                               \
      err = std::string(#call) + ": " + api().errorString(r_);                             \
      return CUSHA_ENCCL;                                                                  \
    }                                                                                      \
  } while (0)
}  // namespace

int nccl_unique_id(void* out128, std::string& err) {
  if (!api().ok) { err = api().why; return CUSHA_EUNSUPPORTED; }
  ncclUniqueId id;
  NC(api().getUniqueId(&id));
  static_assert(sizeof(ncclUniqueId) == 128, "ncclUniqueId is 128 bytes");
  std::memcpy(out128, &id, sizeof(id));
  return CUSHA_OK;
}

int nccl_init(Graph& g, const void* id128, std::string& err) {
  if (!api().ok) { err = api().why; return CUSHA_EUNSUPPORTED; }
  ncclUniqueId id;
  std::memcpy(&id, id128, sizeof(id));
  ncclComm_t comm = nullptr;
  NC(api().commInitRank(&comm, g.world_size, id, g.rank));
  g.nccl_comm = comm;
  return CUSHA_OK;
}

// Each rank r broadcasts its owned slices from the same device buffers (in
// place), so after the group every rank holds every slice.
int nccl_exchange(Graph& g, uint32_t vb, bool final_values, std::string& err) {
  ncclComm_t comm = static_cast<ncclComm_t>(g.nccl_comm);
  NC(api().groupStart());
  for (int r = 0; r < g.world_size; ++r) {
    const uint64_t s0 = g.h_bounds[r], s1 = g.h_bounds[r + 1];
    const uint64_t v0 = std::min<uint64_t>(s0 * g.N, g.V), v1 = std::min<uint64_t>(s1 * g.N, g.V);
    if (final_values) {
      char* vv = static_cast<char*>(g.d_vv);
      NC(api().broadcast(vv + v0 * vb, vv + v0 * vb, (v1 - v0) * vb, ncclUint8, r, comm, g.stream));
    } else {
      NC(api().broadcast(g.d_gathered + v0, g.d_gathered + v0, v1 - v0, ncclUint32, r, comm, g.stream));
      NC(api().broadcast(g.d_active + s0, g.d_active + s0, s1 - s0, ncclUint8, r, comm, g.stream));
    }
  }
  NC(api().groupEnd());
  return CUSHA_OK;
}

void nccl_destroy(Graph& g) {
  if (g.nccl_comm && api().ok) api().commDestroy(static_cast<ncclComm_t>(g.nccl_comm));
  g.nccl_comm = nullptr;
}

}  // namespace cusha
