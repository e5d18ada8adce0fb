// nccl.cu — the multi-GPU exchange of row (e) over NCCL (NVLink 5 / NVSwitch).
//
// libnccl.so.2 is opened at run time (dlopen), so single-GPU use has no NCCL
// dependency; torch ships the library and has normally loaded it already.
// NCCL only bootstraps the ranks: at build time it all-gathers the CUDA IPC
// handles of every rank's SrcValue, dirty[], barrier block and VertexValues.
// Everything after that is peer memory over NVLink / NVSwitch (api.cu,
// kernels.cu): stage 4 stores the write-back values straight into the owning
// rank's SrcValue, the per-pass barrier and convergence vote are stores and
// system-scope atomics into the ranks' barrier blocks, and cusha_get_values
// reads every rank's VertexValues slice directly.
#include <dlfcn.h>
#include <nccl.h>

#include <algorithm>
#include <chrono>
#include <cstring>
#include <thread>
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
  decltype(&ncclCommGetAsyncError) asyncError = nullptr;
  decltype(&ncclCommAbort) commAbort = nullptr;
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
    x.asyncError = reinterpret_cast<decltype(x.asyncError)>(dlsym(h, "ncclCommGetAsyncError"));
    x.commAbort = reinterpret_cast<decltype(x.commAbort)>(dlsym(h, "ncclCommAbort"));
    x.groupStart = reinterpret_cast<decltype(x.groupStart)>(dlsym(h, "ncclGroupStart"));
    x.groupEnd = reinterpret_cast<decltype(x.groupEnd)>(dlsym(h, "ncclGroupEnd"));
    x.errorString = reinterpret_cast<decltype(x.errorString)>(dlsym(h, "ncclGetErrorString"));
    x.ok = x.getUniqueId && x.commInitRank && x.commDestroy && x.broadcast && x.groupStart && x.groupEnd &&
           x.errorString && x.allGather && x.allReduce && x.asyncError && x.commAbort;
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
  if (!g.nccl_comm) { err = "the NCCL communicator was aborted"; return CUSHA_ENCCL; }
  NC(api().allGather(dsend, drecv, bytes, ncclUint8, static_cast<ncclComm_t>(g.nccl_comm), g.stream));
  return CUSHA_OK;
}

// Wait for the work enqueued on g.stream so far without hanging on a failed
// peer: poll the stream and NCCL's asynchronous error state; on an NCCL error
// or after timeout_ms the communicator is aborted (every pending collective
// returns) and CUSHA_ENCCL is returned.
int nccl_wait(Graph& g, uint32_t timeout_ms, std::string& err) {
  cudaEvent_t ev;
  if (cudaEventCreateWithFlags(&ev, cudaEventDisableTiming) != cudaSuccess) { err = "event"; return CUSHA_ECUDA; }
  cudaEventRecord(ev, g.stream);
  const auto t0 = std::chrono::steady_clock::now();
  ncclComm_t comm = static_cast<ncclComm_t>(g.nccl_comm);
  int rc = CUSHA_OK;
  for (;;) {
    const cudaError_t q = cudaEventQuery(ev);
    if (q == cudaSuccess) break;
    if (q != cudaErrorNotReady) { err = std::string("stream: ") + cudaGetErrorString(q); rc = CUSHA_ECUDA; break; }
    ncclResult_t ar = ncclSuccess;
    if (api().asyncError(comm, &ar) != ncclSuccess || (ar != ncclSuccess && ar != ncclInProgress)) {
      err = std::string("NCCL asynchronous error: ") + api().errorString(ar);
      rc = CUSHA_ENCCL;
      break;
    }
    const double ms = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
    if (ms > timeout_ms) {
      err = "NCCL timeout: a rank did not reach the collective within " + std::to_string(timeout_ms) + " ms";
      rc = CUSHA_ENCCL;
      break;
    }
    std::this_thread::sleep_for(std::chrono::microseconds(50));
  }
  cudaEventDestroy(ev);
  if (rc == CUSHA_ENCCL) {
    api().commAbort(comm);
    g.nccl_comm = nullptr;
  }
  return rc;
}

void nccl_destroy(Graph& g) {
  if (g.nccl_comm && api().ok) api().commDestroy(static_cast<ncclComm_t>(g.nccl_comm));
  g.nccl_comm = nullptr;
}

}  // namespace cusha
