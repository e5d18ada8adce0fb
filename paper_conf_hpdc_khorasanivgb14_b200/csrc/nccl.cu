// nccl.cu — the multi-GPU exchange of row (e) over NCCL (NVLink 5 / NVSwitch).
//
// libnccl.so.2 is opened at run time (dlopen), so single-GPU use has no NCCL
// dependency; torch ships the library and has normally loaded it already.
// The write-back values themselves never go through NCCL: stage 4 stores them
// straight into the owning rank's SrcValue over NVLink (CUDA IPC mappings,
// api.cu).  NCCL carries (1) at build time the 64-byte IPC handles of every
// rank's SrcValue / dirty arrays (all-gather), (2) once per pass the
// partition's "committed an update" word (all-reduce MAX), which is both the
// global convergence test of L189 and the barrier between passes, and (3) at
// cusha_get_values every rank's VertexValues slice (grouped broadcasts).
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
  decltype(&ncclAllGather) allGather = nullptr;
  decltype(&ncclAllReduce) allReduce = nullptr;
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
    x.allGather = reinterpret_cast<decltype(x.allGather)>(dlsym(h, "ncclAllGather"));
    x.allReduce = reinterpret_cast<decltype(x.allReduce)>(dlsym(h, "ncclAllReduce"));
    x.groupStart = reinterpret_cast<decltype(x.groupStart)>(dlsym(h, "ncclGroupStart"));
    x.groupEnd = reinterpret_cast<decltype(x.groupEnd)>(dlsym(h, "ncclGroupEnd"));
    x.errorString = reinterpret_cast<decltype(x.errorString)>(dlsym(h, "ncclGetErrorString"));
    x.ok = x.getUniqueId && x.commInitRank && x.commDestroy && x.broadcast && x.groupStart && x.groupEnd &&
           x.errorString && x.allGather && x.allReduce;
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

int nccl_allgather_bytes(Graph& g, const void* dsend, void* drecv, size_t bytes, std::string& err) {
  NC(api().allGather(dsend, drecv, bytes, ncclUint8, static_cast<ncclComm_t>(g.nccl_comm), g.stream));
  return CUSHA_OK;
}

int nccl_allreduce_max_u32(Graph& g, const uint32_t* dsend, uint32_t* drecv, std::string& err) {
  NC(api().allReduce(dsend, drecv, 1, ncclUint32, ncclMax, static_cast<ncclComm_t>(g.nccl_comm), g.stream));
  return CUSHA_OK;
}

// Rank r broadcasts its VertexValues slice (its vertices [v0, v0 + nvl)) into
// the same place of every rank's |V|-element buffer dfull.
int nccl_gather_values(Graph& g, void* dfull, uint32_t vb, std::string& err) {
  ncclComm_t comm = static_cast<ncclComm_t>(g.nccl_comm);
  char* full = static_cast<char*>(dfull);
  NC(api().groupStart());
  for (uint32_t r = 0; r < g.G; ++r) {
    const uint64_t v0 = std::min<uint64_t>((uint64_t)g.h_bounds[r] * g.N, g.V);
    const uint64_t v1 = std::min<uint64_t>((uint64_t)g.h_bounds[r + 1] * g.N, g.V);
    const void* send = r == g.part ? g.d_vv : full + v0 * vb;
    NC(api().broadcast(send, full + v0 * vb, (v1 - v0) * vb, ncclUint8, (int)r, comm, g.stream));
  }
  NC(api().groupEnd());
  return CUSHA_OK;
}

void nccl_destroy(Graph& g) {
  if (g.nccl_comm && api().ok) api().commDestroy(static_cast<ncclComm_t>(g.nccl_comm));
  g.nccl_comm = nullptr;
}

}  // namespace cusha
