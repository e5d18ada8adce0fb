// api.cu — the C ABI of include/cusha.h (row b) and the iteration driver (row a5).
//
// cusha_run replaces the paper's host loop (Fig. 5 lines 0-2 and 29; L189:
// launch, cudaMemcpy(is_converged), decide).  On one GPU the default is ONE
// launch for the whole run (overlapped passes, kernels.cu); the per-pass mode
// launches a fixed-count CUDA graph of passes and checks the device-resident
// convergence flag once per graph.  A destination-range partitioned graph
// (row e) runs one pass per partition, then decides global convergence from
// every partition's "committed an update" word (NCCL all-reduce across GPUs,
// or directly in the one-process simulation).
#include <algorithm>
#include <cmath>
#include <cstring>
#include <string>
#include <vector>

#include <nvtx3/nvToolsExt.h>

#include "algorithms.cuh"
#include "graph.hpp"

namespace cusha {

static thread_local std::string t_err;
void set_error(const std::string& msg) { t_err = msg; }

static int fail(int code, const std::string& msg) {
  set_error(msg);
  return code;
}

#define CKA(call)                                                                                  \
  do {                                                                                             \
    cudaError_t e_ = (call);                                                                       \
    if (e_ != cudaSuccess) {                                                                       \
      return fail(e_ == cudaErrorMemoryAllocation ? CUSHA_ENOMEM : CUSHA_ECUDA,                    \
                  std::string(#call) + ": " + cudaGetErrorString(e_));                             \
    }                                                                                              \
  } while (0)

// one partition; G partitions in this process; one process per GPU
// bootstrapped over NCCL; one process per GPU bootstrapped by the caller
constexpr int kModeSingle = 0, kModeSim = 1, kModeNccl = 2, kModeIpc = 3;
constexpr size_t kIpcBlob = 4 * sizeof(cudaIpcMemHandle_t);  // SrcValue, dirty, barrier block, VertexValues

// NVTX ranges around the ABI calls (SURVEY §5 tracing): header-only NVTX v3,
// free unless a tool (nsys, ncu --nvtx) is attached
struct NvtxRange {
  explicit NvtxRange(const char* name) { nvtxRangePushA(name); }
  ~NvtxRange() { nvtxRangePop(); }
};
constexpr int kChunk = 16;  // passes per fixed-count graph / per host check (per-pass modes)
#ifndef CUSHA_WIDE_WINDOW
#define CUSHA_WIDE_WINDOW 4
#endif
constexpr uint32_t kWideWindow = CUSHA_WIDE_WINDOW, kLowDegree = 4;
constexpr uint32_t kHostTrace = 256;  // trace records read back with the Ctl block (more: a second copy)

// launch configuration of the shard pass for one (graph, algorithm): computed
// once per graph and algorithm (pass_config), reused by every later run
struct PassCfg {
  size_t smem = 0;
  int mapj = 0, stash = 0;
  uint32_t nst = 0;
  uint32_t grid = 0;  // persistent grid (resident CTAs)
  bool one_cta = false;
};

}  // namespace cusha

// The handle: one partition on a single GPU or per rank (NCCL), or all G
// partitions of the one-process simulation (same kernels and layout as the
// per-rank mode; the "peer" SrcValue arrays are the sibling partitions').
struct cusha_graph {
  int mode = cusha::kModeSingle;
  std::vector<cusha::Graph*> parts;
  cudaStream_t stream = nullptr;
  bool own_stream = false;
  int device = 0;
  cudaGraphExec_t exec[cusha::kNumAlgs] = {};  // per-pass mode: kChunk passes per graph (single partition)
  cudaGraphExec_t chunk_exec[cusha::kNumAlgs] = {};  // partitioned / BSP: one captured chunk of rounds
  bool chunk_uncapturable[cusha::kNumAlgs] = {};
  cusha::Ctl** d_ctls = nullptr;                // partitioned: device array of the partitions' Ctl (sim) / own (NCCL)
  cusha_stats st{};
  int last_alg = -1;
  bool have_values = false;
  cusha::PassCfg cfg[cusha::kNumAlgs];  // pass_config per algorithm (valid where cfg_ok)
  bool cfg_ok[cusha::kNumAlgs] = {};
};

namespace cusha {

static uint64_t device_bytes(const Graph& g) {
  uint64_t b = 4ull * (g.Sl + 1) * 2 + 4ull * g.Sl * 2;  // shard / CW offsets + counts
  // per-entry arrays count whole; their host-streamed tails (row f3) are subtracted below
  b += 2 * g.P;                                          // DestIndex
  if (g.d_eid || g.h_eid) b += 4 * g.P;
  if (g.has_ev) b += 4 * g.P;
  if (g.d_srcloc || g.h_srcloc) b += 2 * g.P;
  if (g.d_win) b += 4ull * (g.Sl + 1) * g.S;
  if (g.d_cw_src || g.h_cw_src) b += 2 * g.Q;
  if (g.d_mapper || g.h_mapper) b += 4 * g.Q;
  if (g.d_cw_win || g.h_cw_win) b += 2 * g.Q;
  if (g.d_cw_delta) b += 4ull * g.Sl * g.S;
  if (g.d_cwp) b += 4ull * g.Sl * (g.G + 1) + g.S;
  b += 4ull * g.nvl;                                     // out-degrees
  b += 4 * (g.P + 1) * (g.bsp ? 2 : 1) + 8ull * g.nvl;  // SrcValue (two copies in BSP mode) + VertexValues
  return b - g.host_bytes;                               // minus the host-streamed part (row f3)
}

static void free_handle(cusha_graph* h) {
  if (!h) return;
  cudaSetDevice(h->device);
  for (auto& e : h->exec)
    if (e) cudaGraphExecDestroy(e);
  for (auto& e : h->chunk_exec)
    if (e) cudaGraphExecDestroy(e);
  for (Graph* g : h->parts) {
    free_device_arrays(*g);
    nccl_destroy(*g);
    g->free_mirror();
    for (cudaEvent_t e : {g->ev0, g->evm, g->ev1})
      if (e) cudaEventDestroy(e);
    delete g;
  }
  h->parts.clear();
  if (h->d_ctls) cudaFreeAsync(h->d_ctls, h->stream);
  if (h->own_stream && h->stream) {
    cudaStreamSynchronize(h->stream);
    cudaStreamDestroy(h->stream);
  } else if (h->stream) {
    cudaStreamSynchronize(h->stream);
  }
  delete h;
}

static Graph& g0(cusha_graph* h) { return *h->parts[0]; }
static const Graph& g0(const cusha_graph* h) { return *h->parts[0]; }

// Per-run arrays of a partition: SrcValue (P entries + 1), VertexValues
// (8 B per owned vertex covers every Table-3 Vertex), the control block.
// With one process per GPU, SrcValue and dirty[] are cudaMalloc'ed so the
// other ranks can map them (CUDA IPC) and store into them over NVLink.
static int alloc_run_state(Graph& g, bool ipc) {
  g.srcvalue_ipc = ipc;
  if (ipc) {  // the arrays the other ranks map: SrcValue, dirty[], the barrier block, VertexValues
    CKA(cudaMalloc(&g.d_srcvalue, 4 * (g.P + 1)));
    if (g.skip_clean) {
      if (g.d_dirty) cudaFreeAsync(g.d_dirty, g.stream);
      g.d_dirty = nullptr;
      CKA(cudaMalloc(&g.d_dirty, 4ull * std::max<uint32_t>(g.Sl, 1)));
    }
    CKA(cudaMalloc(&g.d_sync, sizeof(PeerSync)));
    CKA(cudaMemsetAsync(g.d_sync, 0, sizeof(PeerSync), g.stream));
    CKA(cudaMalloc(&g.d_vv, 8ull * std::max<uint32_t>(g.nvl, 1)));
  } else {
    CKA(dev_alloc((void**)&g.d_srcvalue, 4 * (g.P + 1), g.stream));
    CKA(dev_alloc(&g.d_vv, 8ull * std::max<uint32_t>(g.nvl, 1), g.stream));
  }
  CKA(cudaMemsetAsync(g.d_srcvalue, 0, 4 * (g.P + 1), g.stream));
  if (g.bsp) {
    CKA(dev_alloc((void**)&g.d_srcvalue2, 4 * (g.P + 1), g.stream));
    CKA(cudaMemsetAsync(g.d_srcvalue2, 0, 4 * (g.P + 1), g.stream));
  }
  CKA(dev_alloc((void**)&g.d_ctl, sizeof(Ctl), g.stream));
  CKA(cudaMemsetAsync(g.d_ctl, 0, sizeof(Ctl), g.stream));
  // host mirror of the Ctl block and the trace head, read back together at the
  // end of a run.  Pageable on purpose: pinning (cudaMallocHost / cudaFreeHost)
  // per graph costs more than the copy it would save (e2e builds and frees a
  // graph per step)
  struct HostMirror {
    Ctl ctl;
    TraceRec tr[kHostTrace];
  };
  HostMirror* hm = new (std::nothrow) HostMirror();
  if (!hm) return fail(CUSHA_ENOMEM, "host allocation");
  g.h_ctl = &hm->ctl;
  g.h_trace = hm->tr;
  g.h_mirror = hm;
  g.mirror_deleter = [](void* q) { delete static_cast<HostMirror*>(q); };
  CKA(cudaEventCreate(&g.ev0));
  CKA(cudaEventCreate(&g.evm));
  CKA(cudaEventCreate(&g.ev1));
  return CUSHA_OK;
}

// Peer tables of the partitioned mode: SrcValue (and dirty[]) of every
// partition, as device pointers valid on this device.
static int set_peer_tables(Graph& g, const std::vector<uint32_t*>& sv, const std::vector<uint32_t*>& dirty) {
  CKA(dev_alloc((void**)&g.d_sv_peer, sizeof(uint32_t*) * g.G, g.stream));
  CKA(cudaMemcpyAsync(g.d_sv_peer, sv.data(), sizeof(uint32_t*) * g.G, cudaMemcpyHostToDevice, g.stream));
  if (g.skip_clean) {
    CKA(dev_alloc((void**)&g.d_dirty_peer, sizeof(uint32_t*) * g.G, g.stream));
    CKA(cudaMemcpyAsync(g.d_dirty_peer, dirty.data(), sizeof(uint32_t*) * g.G, cudaMemcpyHostToDevice, g.stream));
  }
  CKA(cudaStreamSynchronize(g.stream));  // the host vectors go out of scope
  return CUSHA_OK;
}

// One process per GPU: this rank's CUDA IPC handles (SrcValue, dirty[], the
// barrier block, VertexValues), and the mapping of every other rank's.
static int ipc_export_blob(Graph& g, void* out) {
  cudaIpcMemHandle_t h[4];
  std::memset(h, 0, sizeof(h));
  CKA(cudaIpcGetMemHandle(&h[0], g.d_srcvalue));
  if (g.skip_clean) CKA(cudaIpcGetMemHandle(&h[1], g.d_dirty));
  CKA(cudaIpcGetMemHandle(&h[2], g.d_sync));
  CKA(cudaIpcGetMemHandle(&h[3], g.d_vv));
  std::memcpy(out, h, sizeof(h));
  return CUSHA_OK;
}

static int ipc_connect_blob(Graph& g, const void* all) {
  const uint32_t G = g.G;
  std::vector<cudaIpcMemHandle_t> h(4 * G);
  std::memcpy(h.data(), all, kIpcBlob * G);
  std::vector<uint32_t*> sv(G), dirty(G, nullptr);
  std::vector<PeerSync*> sync(G);
  g.vv_peer.assign(G, nullptr);
  auto open = [&](const cudaIpcMemHandle_t& hd, void** p) -> int {
    CKA(cudaIpcOpenMemHandle(p, hd, cudaIpcMemLazyEnablePeerAccess));
    g.ipc_open.push_back(*p);
    return CUSHA_OK;
  };
  int rc;
  for (uint32_t q = 0; q < G; ++q) {
    if (q == g.part) {
      sv[q] = g.d_srcvalue; dirty[q] = g.d_dirty; sync[q] = g.d_sync; g.vv_peer[q] = g.d_vv;
      continue;
    }
    void* p = nullptr;
    if ((rc = open(h[4 * q], &p))) return rc;
    sv[q] = static_cast<uint32_t*>(p);
    if (g.skip_clean) {
      if ((rc = open(h[4 * q + 1], &p))) return rc;
      dirty[q] = static_cast<uint32_t*>(p);
    }
    if ((rc = open(h[4 * q + 2], &p))) return rc;
    sync[q] = static_cast<PeerSync*>(p);
    if ((rc = open(h[4 * q + 3], &p))) return rc;
    g.vv_peer[q] = p;
  }
  if ((rc = set_peer_tables(g, sv, dirty))) return rc;
  CKA(dev_alloc((void**)&g.d_sync_peer, sizeof(PeerSync*) * G, g.stream));
  CKA(cudaMemcpyAsync(g.d_sync_peer, sync.data(), sizeof(PeerSync*) * G, cudaMemcpyHostToDevice, g.stream));
  CKA(cudaStreamSynchronize(g.stream));
  g.connected = true;
  return CUSHA_OK;
}

// NCCL bootstrap: all-gather every rank's handles, then map them
static int connect_ipc_peers(Graph& g) {
  const uint32_t G = g.G;
  std::vector<uint8_t> mine(kIpcBlob), all(kIpcBlob * G);
  int rc = ipc_export_blob(g, mine.data());
  if (rc) return rc;
  void* dsend = nullptr;
  void* drecv = nullptr;
  CKA(dev_alloc(&dsend, kIpcBlob, g.stream));
  CKA(dev_alloc(&drecv, kIpcBlob * G, g.stream));
  CKA(cudaMemcpyAsync(dsend, mine.data(), kIpcBlob, cudaMemcpyHostToDevice, g.stream));
  std::string err;
  rc = nccl_allgather_bytes(g, dsend, drecv, kIpcBlob, err);
  if (!rc) rc = nccl_wait(g, g.comm_timeout_ms, err);
  if (rc) return fail(rc, "IPC handle exchange: " + err);
  CKA(cudaMemcpyAsync(all.data(), drecv, kIpcBlob * G, cudaMemcpyDeviceToHost, g.stream));
  CKA(cudaStreamSynchronize(g.stream));
  cudaFreeAsync(dsend, g.stream);
  cudaFreeAsync(drecv, g.stream);
  return ipc_connect_blob(g, all.data());
}

}  // namespace cusha

using namespace cusha;

extern "C" {

const char* cusha_last_error(void) { return t_err.c_str(); }
int cusha_abi_version(void) { return CUSHA_ABI_VERSION; }

size_t cusha_value_bytes(cusha_algorithm alg) {
  if ((int)alg < 0 || (int)alg >= kNumAlgs) return 0;
  return value_bytes((int)alg);
}

uint32_t cusha_shard_size(uint32_t V, uint64_t E, uint32_t vertex_bytes, uint32_t smem_per_sm,
                          uint32_t reserved_per_block) {
  // L310: |N| such that the average window |E||N|^2/|V|^2 (L173) is 32, then
  // snapped to the nearest size that uses a whole share of the SM's shared memory.
  if (V == 0) return 1;
  if (vertex_bytes == 0) vertex_bytes = 4;
  if (smem_per_sm == 0) {  // B200 defaults: 228 KB per SM, 1 KB reserved per resident CTA
    smem_per_sm = 233472;
    reserved_per_block = 1024;
  }
  double n0 = E ? (double)V * std::sqrt(32.0 / (double)E) : (double)V;
  uint32_t best = 0;
  double bestd = 1e300;
  for (uint32_t k = 1; k <= 32; ++k) {
    const int64_t q = (int64_t)(smem_per_sm / k) - (int64_t)reserved_per_block;
    if (q <= 0) continue;
    uint64_t nk = (uint64_t)q / vertex_bytes;
    if (nk > 65534) nk = 65534;
    if (nk == 0) continue;
    const double d = std::fabs((double)nk - n0);
    if (d < bestd) { bestd = d; best = (uint32_t)nk; }
  }
  if (best == 0) best = 1;
  if (best > V) best = V;
  return best;
}

int cusha_build_graph(uint32_t V, uint64_t E, const uint32_t* src, const uint32_t* dst, const uint32_t* edge_values,
                      const cusha_build_opts* opts, cusha_graph** out) {
  if (!out) return fail(CUSHA_EINVAL, "out is NULL");
  NvtxRange nvtx("cusha_build_graph");
  *out = nullptr;
  if (V == 0) return fail(CUSHA_EINVAL, "num_vertices must be > 0");
  if (V >= (1u << 31)) return fail(CUSHA_EINVAL, "num_vertices must be < 2^31");
  if (E >= 0xFFFFFFFFull - (1ull << 26)) return fail(CUSHA_EINVAL, "num_edges too large for 32-bit positions");
  if (E && (!src || !dst)) return fail(CUSHA_EINVAL, "src/dst are NULL");
  cusha_build_opts o{};
  if (opts) o = *opts;
  if (o.repr != CUSHA_REPR_GSHARDS && o.repr != CUSHA_REPR_CW) return fail(CUSHA_EINVAL, "bad repr");
  if (o.world_size <= 0) o.world_size = 1;
  if (o.world_size > 64) return fail(CUSHA_EINVAL, "world_size must be <= 64");
  if (o.world_size > 1 && o.repr != CUSHA_REPR_CW)
    return fail(CUSHA_EUNSUPPORTED, "the partitioned (multi-GPU) mode uses the CW representation");
  if (o.transport != CUSHA_TRANSPORT_NCCL && o.transport != CUSHA_TRANSPORT_IPC)
    return fail(CUSHA_EINVAL, "transport must be NCCL or IPC");
  const bool multiproc = o.world_size > 1 && (o.nccl_unique_id || o.transport == CUSHA_TRANSPORT_IPC);
  if (multiproc && (o.rank < 0 || o.rank >= o.world_size)) return fail(CUSHA_EINVAL, "rank out of range");
  uint32_t N = o.vertices_per_shard ? o.vertices_per_shard : cusha_shard_size(V, E, o.smem_bytes_per_vertex, 0, 0);
  if (N > 65534) return fail(CUSHA_EINVAL, "vertices_per_shard must be <= 65534");
  if (o.pass_barrier < 0 || o.pass_barrier > 2) return fail(CUSHA_EINVAL, "pass_barrier must be 0, 1 or 2");
  if (o.mode != CUSHA_MODE_ASYNC && o.mode != CUSHA_MODE_BSP) return fail(CUSHA_EINVAL, "mode must be ASYNC or BSP");
  if (o.mode == CUSHA_MODE_BSP && o.world_size > 1)
    return fail(CUSHA_EUNSUPPORTED, "the two-phase BSP mode runs one partition");
  if (N > V) N = V;
  const uint32_t S = (V + N - 1) / N;
  const int mode = o.world_size == 1 ? kModeSingle
                   : o.transport == CUSHA_TRANSPORT_IPC ? kModeIpc
                   : (o.nccl_unique_id ? kModeNccl : kModeSim);
  const uint32_t G = std::min<uint32_t>((uint32_t)o.world_size, S);  // never more partitions than shards
  if (multiproc && G != (uint32_t)o.world_size) return fail(CUSHA_EINVAL, "world_size exceeds the number of shards");

  cusha_graph* h = new (std::nothrow) cusha_graph();
  if (!h) return fail(CUSHA_ENOMEM, "host allocation");
  h->mode = G > 1 ? mode : kModeSingle;
  h->device = o.device;
  auto bail = [&](int code) { free_handle(h); return code; };
  auto cu = [&](cudaError_t e, const char* what) -> int {
    if (e == cudaSuccess) return 0;
    set_error(std::string(what) + ": " + cudaGetErrorString(e));
    return e == cudaErrorMemoryAllocation ? CUSHA_ENOMEM : CUSHA_ECUDA;
  };
  int rc;
  if ((rc = cu(cudaSetDevice(o.device), "cudaSetDevice"))) return bail(rc);
  if (o.stream) {
    h->stream = (cudaStream_t)o.stream;
  } else {
    if ((rc = cu(cudaStreamCreateWithFlags(&h->stream, cudaStreamNonBlocking), "cudaStreamCreate"))) return bail(rc);
    h->own_stream = true;
  }
  Graph* glob = new (std::nothrow) Graph();
  if (!glob) return bail(fail(CUSHA_ENOMEM, "host allocation"));
  h->parts.push_back(glob);  // freed with the handle on any failure
  Graph& g = *glob;
  g.V = V; g.E = E; g.N = N; g.S = S; g.repr = (int)o.repr; g.device = o.device; g.stream = h->stream;
  g.host_loop = o.host_loop != 0;
  g.skip_clean = o.skip_clean_shards != 0;
  g.pass_barrier = o.pass_barrier;
  g.topo_budget = o.device_topology_budget;
  g.keep_ids = o.keep_layout != 0;
  g.bsp = o.mode == CUSHA_MODE_BSP;
  g.world_size = o.world_size;
  g.rank = multiproc ? o.rank : 0;
  cudaEvent_t e0 = nullptr, eh = nullptr, e1 = nullptr;
  if ((rc = cu(cudaEventCreate(&e0), "cudaEventCreate")) || (rc = cu(cudaEventCreate(&eh), "cudaEventCreate")) ||
      (rc = cu(cudaEventCreate(&e1), "cudaEventCreate")))
    return bail(rc);
  struct EvGuard {
    cudaEvent_t a, b, c;
    ~EvGuard() { cudaEventDestroy(a); cudaEventDestroy(b); cudaEventDestroy(c); }
  } evg{e0, eh, e1};

  CKA(cudaEventRecord(e0, h->stream));
  const uint32_t *d_src = src, *d_dst = dst, *d_val = edge_values;
  void* tmp = nullptr;
  uint64_t h2d = 0;
  InputChunks chunks;
  cudaStream_t cs = nullptr;  // copy stream of the host-input path (row f2)
  struct CopyGuard {
    InputChunks* c;
    cudaStream_t* s;
    ~CopyGuard() {
      if (*s) { cudaStreamSynchronize(*s); cudaStreamDestroy(*s); }
      for (int i = 0; i < c->n; ++i) cudaEventDestroy(c->ready[i]);
      if (c->all) cudaEventDestroy(c->all);
    }
  } cg{&chunks, &cs};
  if (h->mode == kModeSingle && o.input_location == CUSHA_INPUT_HOST && E) {
    // the host edge list crosses in chunks on a copy stream; the layout's first
    // pass (keys, degrees) consumes each chunk as it lands (DESIGN.md f2)
    const uint64_t nvals = edge_values ? 3 : 2;
    if ((rc = cu(dev_alloc(&tmp, nvals * E * 4, h->stream), "cudaMallocAsync(inputs)"))) return bail(rc);
    uint32_t* t = static_cast<uint32_t*>(tmp);
    if ((rc = cu(cudaStreamCreateWithFlags(&cs, cudaStreamNonBlocking), "cudaStreamCreate(copy)")) ||
        (rc = cu(cudaEventRecord(eh, h->stream), "event"))) {  // the allocation precedes the copies
      cudaFreeAsync(tmp, h->stream);
      return bail(rc);
    }
    chunks.n = E >= (1ull << 22) ? 8 : 1;
    if (const char* v = std::getenv("CUSHA_H2D_CHUNKS"))  // tuning probe only
      if (E >= (1ull << 22)) chunks.n = std::max(1, std::min(16, std::atoi(v)));
    for (int c = 0; c <= chunks.n; ++c)  // inner bounds on 256-edge boundaries (aligned chunk sorts)
      chunks.bounds[c] = c == chunks.n ? E : (E * (uint64_t)c / (uint64_t)chunks.n) & ~255ull;
    rc = cu(cudaStreamWaitEvent(cs, eh, 0), "wait");
    for (int c = 0; c < chunks.n && !rc; ++c) {
      const uint64_t lo = chunks.bounds[c], n = chunks.bounds[c + 1] - lo;
      if ((rc = cu(cudaEventCreateWithFlags(&chunks.ready[c], cudaEventDisableTiming), "event")) ||
          (rc = cu(cudaMemcpyAsync(t + lo, src + lo, n * 4, cudaMemcpyHostToDevice, cs), "H2D src")) ||
          (rc = cu(cudaMemcpyAsync(t + E + lo, dst + lo, n * 4, cudaMemcpyHostToDevice, cs), "H2D dst")) ||
          (rc = cu(cudaEventRecord(chunks.ready[c], cs), "event")))
        break;
    }
    if (!rc && edge_values)
      rc = cu(cudaMemcpyAsync(t + 2 * E, edge_values, E * 4, cudaMemcpyHostToDevice, cs), "H2D values");
    if (!rc && !(rc = cu(cudaEventCreate(&chunks.all), "event"))) rc = cu(cudaEventRecord(chunks.all, cs), "event");
    if (rc) {
      cudaStreamSynchronize(cs);
      cudaFreeAsync(tmp, h->stream);
      return bail(rc);
    }
    d_src = t; d_dst = t + E; d_val = edge_values ? t + 2 * E : nullptr;
    h2d = nvals * E * 4;
  }
  std::string err;
  if (h->mode == kModeSingle) {
    rc = build_layout(g, d_src, d_dst, d_val, err, chunks.n ? &chunks : nullptr);
    if (tmp) cudaFreeAsync(tmp, h->stream);  // stream order: the build waited for every copy
    if (rc) {
      set_error("build: " + err);
      return bail(rc);
    }
  }
  if (h->mode == kModeSingle) {
    // CW reads no window table after the build (unless skipping clean shards or inspecting the layout)
    if (g.repr == CUSHA_REPR_CW && !g.skip_clean && !g.keep_ids && g.d_win) {
      cudaFreeAsync(g.d_win, h->stream);
      g.d_win = nullptr;
    }
    g.h_bounds = {0u, S};
    rc = offload_topology(g, err);  // row f3 (no-op without a budget)
    if (rc) {
      set_error("host topology: " + err);
      return bail(rc);
    }
    if ((rc = alloc_run_state(g, false))) return bail(rc);
  } else {
    // destination-range partition (row e): the shard-pair counts place the
    // bounds (near-equal work); each partition then sorts only its own in- and
    // out-edges, streamed from wherever the edge list lives (partition.cu)
    PlanInput pin;
    pin.V = V; pin.N = N; pin.E = E; pin.src = src; pin.dst = dst; pin.val = edge_values;
    pin.host = o.input_location == CUSHA_INPUT_HOST; pin.stream = h->stream;
    Plan plan;
    struct PlanGuard {
      Plan* p;
      cudaStream_t s;
      ~PlanGuard() { free_plan(*p, s); }
    } pgd{&plan, h->stream};
    if ((rc = plan_partitions(pin, G, plan, err))) {
      set_error("partition: " + err);
      return bail(rc);
    }
    if (plan.bounds.size() - 1 != G) return bail(fail(CUSHA_EINVAL, "partition count"));
    std::vector<Graph*> parts;
    const bool ranked = h->mode == kModeNccl || h->mode == kModeIpc;  // this process holds its rank's partition
    const uint32_t r0 = ranked ? (uint32_t)o.rank : 0u, r1 = ranked ? r0 + 1 : G;
    for (uint32_t r = r0; r < r1; ++r) {
      Graph* p = new (std::nothrow) Graph();
      if (!p) { for (Graph* x : parts) { free_device_arrays(*x); delete x; } return bail(fail(CUSHA_ENOMEM, "host")); }
      parts.push_back(p);
      p->device = o.device; p->stream = h->stream; p->skip_clean = g.skip_clean; p->host_loop = true;
      p->pass_barrier = 1; p->world_size = o.world_size; p->rank = (int)r; p->keep_ids = g.keep_ids;
      if ((rc = build_part_direct(pin, plan, r, *p, err))) {
        for (Graph* x : parts) { free_device_arrays(*x); delete x; }
        set_error("partition: " + err);
        return bail(rc);
      }
      if (!p->skip_clean && !p->keep_ids && p->d_win) {  // only the clean-shard marks read the window rows
        cudaFreeAsync(p->d_win, h->stream);
        p->d_win = nullptr;
      }
      // row f3: the partition's per-entry topology beyond the budget goes to
      // pinned host memory now, before the next partition's build needs HBM
      p->topo_budget = g.topo_budget;
      if ((rc = offload_topology(*p, err))) {
        for (Graph* x : parts) { free_device_arrays(*x); delete x; }
        set_error("host topology: " + err);
        return bail(rc);
      }
    }
    if (pin.host) h2d = (1 + 2ull * (r1 - r0)) * (edge_values ? 3 : 2) * 4 * E;  // the streamed passes
    // the handle now holds the partitions
    free_device_arrays(g);
    delete glob;
    h->parts = parts;
    for (Graph* p : h->parts)
      if ((rc = alloc_run_state(*p, ranked))) return bail(rc);
    if (h->mode == kModeSim) {
      std::vector<uint32_t*> sv(G), dirty(G);
      std::vector<Ctl*> ctls(G);
      for (uint32_t q = 0; q < G; ++q) {
        sv[q] = h->parts[q]->d_srcvalue;
        dirty[q] = h->parts[q]->d_dirty;
        ctls[q] = h->parts[q]->d_ctl;
      }
      for (Graph* p : h->parts)
        if ((rc = set_peer_tables(*p, sv, dirty))) return bail(rc);
      CKA(dev_alloc((void**)&h->d_ctls, sizeof(Ctl*) * G, h->stream));
      CKA(cudaMemcpyAsync(h->d_ctls, ctls.data(), sizeof(Ctl*) * G, cudaMemcpyHostToDevice, h->stream));
      CKA(cudaStreamSynchronize(h->stream));
    } else {
      // one process per GPU: the ranks map each other's arrays (CUDA IPC) -
      // over an NCCL all-gather of the handles here, or (transport IPC) by the
      // caller through cusha_ipc_export / cusha_ipc_connect
      Graph& p = *h->parts[0];
      p.comm_timeout_ms = o.comm_timeout_ms ? o.comm_timeout_ms : 300000u;
      if (h->mode == kModeNccl) {
        if ((rc = nccl_init(p, o.nccl_unique_id, err))) {
          set_error("NCCL: " + err);
          return bail(rc);
        }
        if ((rc = connect_ipc_peers(p))) return bail(rc);
      }
    }
  }
  CKA(cudaEventRecord(e1, h->stream));
  CKA(cudaEventSynchronize(e1));
  float ms = 0, ms_h2d = 0;
  cudaEventElapsedTime(&ms, e0, e1);
  if (chunks.all) cudaEventElapsedTime(&ms_h2d, e0, chunks.all);  // build start to the last copy landing
  cusha_stats& st = h->st;
  st.num_vertices = V;
  st.num_edges = E;
  st.vertices_per_shard = N;
  st.num_shards = S;
  st.repr = (uint32_t)o.repr;
  st.last_algorithm = -1;
  st.build_ms = ms;
  st.h2d_ms = ms_h2d;
  st.h2d_bytes = h2d;
  st.world_size = o.world_size;
  st.rank = multiproc ? o.rank : 0;
  st.partitions = h->mode == kModeSingle ? 1 : G;
  st.max_in_degree = g0(h).max_indeg;
  st.device_bytes = 0;
  st.max_part_device_bytes = 0;
  st.entries_padded = 0;
  for (Graph* p : h->parts) {
    p->st = cusha_stats{};
    const uint64_t b = device_bytes(*p);
    st.device_bytes += b;
    st.max_part_device_bytes = std::max(st.max_part_device_bytes, b);
    st.entries_padded += p->P;
  }
  st.host_bytes = 0;
  for (Graph* p : h->parts) st.host_bytes += p->host_bytes;
  st.host_shard = g0(h).host_shard;
  *out = h;
  set_error("");
  return CUSHA_OK;
}

void cusha_free_graph(cusha_graph* h) { free_handle(h); }

int cusha_trim_memory(int device) {
  CKA(cudaSetDevice(device));
  CKA(cudaDeviceSynchronize());
  CKA(trim_pool(device));
  return CUSHA_OK;
}

int cusha_set_vertex_values(cusha_graph* h, cusha_algorithm alg, const void* init, size_t bytes) {
  if (!h || !init) return fail(CUSHA_EINVAL, "null argument");
  if ((int)alg < 0 || (int)alg >= kNumAlgs) return fail(CUSHA_EINVAL, "bad algorithm");
  const uint32_t V = h->st.num_vertices;
  const size_t vb = value_bytes((int)alg);
  const size_t want = (size_t)V * vb;
  if (bytes != want) return fail(CUSHA_EINVAL, "bytes must be |V| * value_bytes(alg)");
  // largest |value| of the field stage 2 reads (fixed-point range, include/cusha.h)
  float mx = 0.f;
  const float* f = static_cast<const float*>(init);
  const size_t stride = vb / 4;
  for (size_t v = 0; v < V; ++v) {
    const float x = std::fabs(f[v * stride]);
    if (!(x <= 3.0e38f)) { mx = INFINITY; break; }
    mx = std::max(mx, x);
  }
  CKA(cudaSetDevice(h->device));
  for (Graph* g : h->parts) {
    const size_t n = (size_t)g->nvl * vb;
    if (!g->d_init[alg]) CKA(dev_alloc(&g->d_init[alg], std::max<size_t>(n, 1), h->stream));
    if (n) CKA(cudaMemcpyAsync(g->d_init[alg], static_cast<const char*>(init) + (size_t)g->v0 * vb, n,
                               cudaMemcpyHostToDevice, h->stream));
    g->init_max_abs[alg] = mx;
  }
  CKA(cudaStreamSynchronize(h->stream));
  return CUSHA_OK;
}

}  // extern "C"

namespace cusha {

// Persistent grid of the shard pass: as many CTAs as fit on the device at
// once (occupancy x SMs), never more than the partition has shards.
static uint32_t pass_grid(const Graph& g, const PassKernel& pk, size_t smem) {
  if (!pk.persistent) return std::max<uint32_t>(g.Sl, 1);
  int sms = 148, per_sm = 1;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, g.device);
  if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, pk.func, (int)pk.threads, smem) != cudaSuccess ||
      per_sm < 1)
    per_sm = 1;
  const uint64_t gsz = (uint64_t)sms * (uint64_t)per_sm;
  return (uint32_t)std::max<uint64_t>(1, std::min<uint64_t>(gsz, g.Sl));
}

// Shared memory of the pass and the CW Mapper form (DESIGN.md "Mapper in
// window form"): the window form (SrcIndexCW + u16 window index per entry, the
// shard's delta row in shared memory) whenever the row fits without lowering
// the CTAs per SM; otherwise the u32 Mapper.  Sets the kernel attributes.
#ifndef CUSHA_MAPJ
#define CUSHA_MAPJ 1  // 0: always the u32 Mapper (tuning comparison)
#endif
#ifndef CUSHA_DEEP_RING
#define CUSHA_DEEP_RING 1  // 0: always the default ring depth (tuning comparison)
#endif
#ifndef CUSHA_FEW_TICKETS
#define CUSHA_FEW_TICKETS 1.25  // below this many shards per resident CTA, run one CTA per SM with a deep ring
#endif
#ifndef CUSHA_STASH
#define CUSHA_STASH 1  // 0: stage 3 of the integer algorithms re-reads VertexValues (tuning comparison)
#endif
static int pass_config(const Graph& g, const PassKernel& pk, PassCfg* c) {
  cudaFuncAttributes fa{};
  CKA(cudaFuncGetAttributes(&fa, pk.func));
  const size_t kMaxSmem = 227 * 1024 - fa.sharedSizeBytes;  // dynamic part of the 227 KB per-CTA limit
  const size_t sm_m = pk.smem_bytes(g.N);
  if (sm_m > kMaxSmem)
    return fail(CUSHA_EINVAL, "vertices_per_shard too large for this algorithm's shared-memory state");
  CKA(cudaFuncSetAttribute(pk.func, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kMaxSmem));
  CKA(cudaFuncSetAttribute(pk.func, cudaFuncAttributePreferredSharedMemoryCarveout, cudaSharedmemCarveoutMaxShared));
  c->smem = sm_m;
  c->mapj = 0;
  const size_t sm_j = pk.smem_bytes(g.N, g.S);
  // ... and only when the rows cost less traffic than they save: an active
  // shard reads its 4|S|-byte row, so |S| rows per pass (4|S|^2 bytes) against
  // 2 bytes per CW entry (|Q| entries) saved over the u32 Mapper
  const bool row_pays = 4ull * g.Sl * g.S <= (uint64_t)g.Q;
  if (CUSHA_MAPJ && row_pays && g.repr == CUSHA_REPR_CW && g.d_cw_win && g.d_cw_delta && !kernels_rle() &&
      g.S <= 0xFFFFu && sm_j <= kMaxSmem) {
    int occ_m = 0, occ_j = 0;
    CKA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ_m, pk.func, (int)pk.threads, sm_m));
    CKA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ_j, pk.func, (int)pk.threads, sm_j));
    if (occ_j >= occ_m && occ_j > 0) {
      c->smem = sm_j;
      c->mapj = 1;
    }
  }
  if (g.repr == CUSHA_REPR_CW && !c->mapj && !g.d_mapper && !g.h_mapper)
    return fail(CUSHA_EUNSUPPORTED, "this graph keeps only the window-form Mapper, whose delta row does not fit");
  // integer algorithms: keep the shard's VertexValues from stage 1 in shared
  // memory for stage 3's update_condition (no second global read) whenever
  // that costs no CTAs per SM
  c->stash = 0;
  const size_t sm_s = c->smem + 4ull * g.N;
  if (CUSHA_STASH && pk.monotone && sm_s <= kMaxSmem) {
    int occ_0 = 0, occ_s = 0;
    CKA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ_0, pk.func, (int)pk.threads, c->smem));
    CKA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ_s, pk.func, (int)pk.threads, sm_s));
    if (occ_s >= occ_0 && occ_s > 0) {
      c->smem = sm_s;
      c->stash = 1;
    }
  }
  // a deeper TMA ring whenever another slot fits at the same CTAs per SM
  // (more bytes in flight per SM; e.g. C5 at one CTA per SM).  With few
  // shards per resident CTA (a pass is about one ticket per CTA, C4) the ring
  // takes the whole SM instead: one CTA per SM, up to 6 slots.  Half as many
  // shards then run at once, so more of them see write-backs made earlier in
  // the same pass (L45) and the run needs fewer passes, while the deep ring
  // keeps the SM's bytes in flight (C4 CC 0.59 -> 0.48 ms)
  c->nst = pk.ring_bytes / pk.slot_bytes;
  if (CUSHA_DEEP_RING) {
    int occ_0 = 0, sms = 148;
    CKA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ_0, pk.func, (int)pk.threads, c->smem));
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, g.device);
    c->one_cta = occ_0 >= 2 && (double)g.Sl < CUSHA_FEW_TICKETS * occ_0 * sms;
    while (c->nst < pk.max_stages && c->smem + pk.slot_bytes <= kMaxSmem) {
      int occ_d = 0;
      CKA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ_d, pk.func, (int)pk.threads, c->smem + pk.slot_bytes));
      if ((occ_d < occ_0 && !c->one_cta) || occ_d == 0) break;
      c->smem += pk.slot_bytes;
      ++c->nst;
    }
  }
  c->grid = pass_grid(g, pk, c->smem);
  return CUSHA_OK;
}

// L2 prefetch of stage-2 tiles beyond the ring (KParams::ahead) pays when a
// pass streams from HBM; on passes that stay in L2 it only adds producer
// latency: on when the entry streams of one pass
// exceed twice the L2.
static int pass_ahead(const Graph& g, int alg) {
  int l2 = 0;
  if (cudaDeviceGetAttribute(&l2, cudaDevAttrL2CacheSize, g.device) != cudaSuccess || l2 <= 0) l2 = 126 << 20;
  // stage 2: SrcValue + DestIndex (+ EdgeValue); stage 4: GS SrcIndex, CW SrcIndexCW + Mapper form
  const uint64_t bytes = (uint64_t)g.P * (6 + (alg_needs_edge_values(alg) ? 4 : 0) + (g.repr == CUSHA_REPR_GSHARDS ? 2 : 0)) +
                         (uint64_t)g.Q * 8;
  return bytes > 2ull * (uint64_t)l2 ? 1 : 0;
}

// Ticket order.  A pass that stays in L2 (no read-ahead) is bound by its
// slowest shards' latency, so it takes the largest shards first; a pass that
// streams from HBM keeps shard order (neighbouring shards share SrcValue lines
// in L2: largest-first was slower on C2, DESIGN.md tuning log v4).
#ifndef CUSHA_BIG_FIRST
#define CUSHA_BIG_FIRST 1
#endif
static int shard_order(Graph& g) {
  if (g.d_order || !g.Sl) return CUSHA_OK;
  std::vector<uint32_t> cnt(g.Sl), ccnt(g.Sl), ord(g.Sl);
  CKA(cudaMemcpyAsync(cnt.data(), g.d_shard_cnt, 4ull * g.Sl, cudaMemcpyDeviceToHost, g.stream));
  CKA(cudaMemcpyAsync(ccnt.data(), g.d_cw_cnt, 4ull * g.Sl, cudaMemcpyDeviceToHost, g.stream));
  CKA(cudaStreamSynchronize(g.stream));
  for (uint32_t s = 0; s < g.Sl; ++s) ord[s] = s;
  std::stable_sort(ord.begin(), ord.end(), [&](uint32_t a, uint32_t b) {
    return (uint64_t)cnt[a] + ccnt[a] > (uint64_t)cnt[b] + ccnt[b];
  });
  CKA(dev_alloc((void**)&g.d_order, 4ull * g.Sl, g.stream));
  CKA(cudaMemcpyAsync(g.d_order, ord.data(), 4ull * g.Sl, cudaMemcpyHostToDevice, g.stream));
  CKA(cudaStreamSynchronize(g.stream));
  return CUSHA_OK;
}

// Chunk table of the one-partition CW SrcValue initialisation
// (init_srcvalue_cw_flat): (shard, first CW position) per kInitChunk entries
// of every CW_i.  Built once per graph, on the first run.
static int init_chunks(Graph& g) {
  if (g.d_init_chunks || g.repr != CUSHA_REPR_CW || g.G != 1 || !g.Sl) return CUSHA_OK;
  std::vector<uint32_t> off(g.Sl), cnt(g.Sl);
  CKA(cudaMemcpyAsync(off.data(), g.d_cw_off, 4ull * g.Sl, cudaMemcpyDeviceToHost, g.stream));
  CKA(cudaMemcpyAsync(cnt.data(), g.d_cw_cnt, 4ull * g.Sl, cudaMemcpyDeviceToHost, g.stream));
  CKA(cudaStreamSynchronize(g.stream));
  std::vector<uint2> ch;
  for (uint32_t s = 0; s < g.Sl; ++s)
    for (uint64_t k = 0; k < cnt[s]; k += kInitChunk) ch.push_back(make_uint2(s, off[s] + (uint32_t)k));
  CKA(dev_alloc((void**)&g.d_init_chunks, sizeof(uint2) * std::max<size_t>(ch.size(), 1), g.stream));
  if (!ch.empty())
    CKA(cudaMemcpyAsync(g.d_init_chunks, ch.data(), sizeof(uint2) * ch.size(), cudaMemcpyHostToDevice, g.stream));
  CKA(cudaStreamSynchronize(g.stream));
  g.init_nchunks = (uint32_t)ch.size();
  return CUSHA_OK;
}

static KParams pass_params(const Graph& g, uint32_t source, const PassCfg& c, int alg) {
  KParams kp = make_params(g, source);
  kp.mapj = c.mapj;
  kp.stash = c.stash;
  kp.nst = c.nst;
  {  // one CTA per SM (the few-tickets mode, or shared memory for one only)
    int sms = 148;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, g.device);
    kp.s4two = c.grid <= (uint32_t)sms ? 1u : 0u;
  }
  kp.ahead = pass_ahead(g, alg);
  if (CUSHA_BIG_FIRST && !kp.ahead) kp.order = g.d_order;
  return kp;
}

// Per-pass mode on one partition: a CUDA graph of kChunk pass launches (no
// conditional node); a pass launched after convergence or max_iters exits at
// once, so the host launches the graph until the flag says stop.
static int ensure_exec(cusha_graph* h, int alg, const PassKernel& pk, const PassCfg& c) {
  if (h->exec[alg]) return CUSHA_OK;
  Graph& g = g0(h);
  cudaGraph_t graph = nullptr;
  CKA(cudaGraphCreate(&graph, 0));
  KParams kp = pass_params(g, 0, c, alg);
  void* args[] = {&kp};
  cudaKernelNodeParams knp = {};
  knp.func = const_cast<void*>(pk.func);
  knp.gridDim = dim3(c.grid);
  knp.blockDim = dim3(pk.threads);
  knp.sharedMemBytes = (unsigned)c.smem;
  knp.kernelParams = args;
  cudaGraphNode_t prev = nullptr, kn;
  cudaError_t e = cudaSuccess;
  for (int i = 0; i < kChunk && e == cudaSuccess; ++i) {
    e = cudaGraphAddKernelNode(&kn, graph, prev ? &prev : nullptr, prev ? 1 : 0, &knp);
    prev = kn;
  }
  if (e == cudaSuccess) e = cudaGraphInstantiate(&h->exec[alg], graph, 0);
  cudaGraphDestroy(graph);
  if (e != cudaSuccess) {
    h->exec[alg] = nullptr;
    return fail(CUSHA_ECUDA, std::string("graph: ") + cudaGetErrorString(e));
  }
  return CUSHA_OK;
}

// Fixed-point range of the float algorithms' stage-2 sums (include/cusha.h):
// every |sum| must stay below 2^31.  PR: sum_{u->v} Rank_u/NbrsNum_u <=
// sum_u Rank_u <= |V| < 2^31 at every pass (the total rank starts at |V| and
// (1-d)|V| + d*(sum over non-dangling) keeps it there).  NN / HS / CS: a
// bound from the initial values, the edge values and the largest in-degree.
static int check_fixed_range(const Graph& g, int a) {
  if (a != kNN && a != kHS && a != kCS) return CUSHA_OK;
  const double w = g.max_abs_ev, x = g.init_max_abs[a], deg = std::max<uint32_t>(g.max_indeg, 1);
  double term = 0;
  if (a == kNN) term = std::max(x, 1.0) * w;       // |x_u * w|, |x_u| <= max(|x0|, 1) after tanh
  else if (a == kHS) term = 2.0 * x * w;            // |(Q_u - Q_v) * coeff|
  else term = std::max(x, 1.0) * std::max(w, 1.0);  // |V_u * G| and G itself
  if (!(term * deg < 2147483648.0))
    return fail(CUSHA_EINVAL, "values x edge values x in-degree reach the 2^31 fixed-point range of the stage-2 sums");
  return CUSHA_OK;
}

static void account_run(const Graph& g, int a, const Ctl& c, bool multi, bool mapj, cusha_stats& st,
                        std::vector<TraceRec>& tr) {
  const uint64_t vb = value_bytes(a);
  const uint64_t evb = alg_needs_edge_values(a) ? 4 : 0;
  const uint32_t n = std::min(c.iter, g.trace_cap);
  uint64_t bytes = 0, paper = 0, edges = 0, wbe = 0, nvp = 0, upd = 0;
  // paper-layout bytes: stage 2 per edge 8 (BFS, CC) / 12 (SSSP, SSWP, NN, PR) / 16 (HS, CS);
  // stage 4 per active edge CW 12 / GS 8 (+4 for 8-byte vertices); stages 1+3 per vertex 2 * sizeof(Vertex)
  const uint64_t p2 = (a == kBFS || a == kCC) ? 8 : (vb == 8 ? 16 : 12);
  const uint64_t p4 = (g.repr == CUSHA_REPR_CW ? 12 : 8) + (vb == 8 ? 4 : 0);
  for (uint32_t i = 0; i < n; ++i) {
    // vertices of the processed shards (all of the partition's unless clean shards were skipped)
    const uint64_t nv = std::min<uint64_t>(g.nvl, tr[i].shards * (uint64_t)g.N);
    bytes += nv * vb + (a == kPR ? 4ull * nv : 0);                    // stages 1+3 reads
    bytes += (uint64_t)tr[i].updated * vb;                            // stage 3 commits
    bytes += tr[i].edges * (4 + 2 + evb);                             // stage 2
    edges += tr[i].edges;
    wbe += tr[i].wb_entries;
    nvp += nv;
    upd += tr[i].updated;
    if (g.repr == CUSHA_REPR_CW)  // SrcIndexCW + window index (+ delta row) or u32 Mapper; SrcValue
      bytes += tr[i].wb_entries * (mapj ? 4 : 6) + tr[i].wb_stores * 4 +
               (mapj ? (uint64_t)tr[i].shards * 4ull * g.S : 0);
    else
      bytes += tr[i].wb_entries * 4 + tr[i].wb_stores * 4 + (uint64_t)tr[i].active_shards * 8ull * g.S;
    paper += tr[i].edges * p2 + tr[i].wb_entries * p4 + nv * 2 * vb;
  }
  st.iterations = c.iter;
  st.converged = c.converged;
  st.algorithmic_bytes = bytes;
  st.paper_bytes = paper;
  st.edges_processed = n == c.iter ? edges : (uint64_t)c.iter * g.E_loc;
  st.wb_entries = wbe;
  st.vertices_processed = nvp;
  st.updated_total = upd;
  st.stage2_bytes_per_iter = g.E_loc * (4 + 2 + evb);
  st.wb_bytes_all_active = g.repr == CUSHA_REPR_CW ? g.E_loc * (mapj ? 8 : 10) : g.E_loc * 8;
  st.mapper_form = (uint32_t)mapj;
  (void)multi;
}

static int read_trace(const Graph& g, uint32_t n, std::vector<TraceRec>& tr) {
  tr.assign(std::max<uint32_t>(n, 1), TraceRec{});
  if (n) {
    CKA(cudaMemcpyAsync(tr.data(), g.d_trace, sizeof(TraceRec) * n, cudaMemcpyDeviceToHost, g.stream));
    CKA(cudaStreamSynchronize(g.stream));
  }
  return CUSHA_OK;
}

}  // namespace cusha

extern "C" {

int cusha_run(cusha_algorithm alg, cusha_graph* h, uint32_t source, uint32_t max_iters) {
  if (!h) return fail(CUSHA_EINVAL, "graph is NULL");
  if ((int)alg < 0 || (int)alg >= kNumAlgs) return fail(CUSHA_EINVAL, "bad algorithm");
  NvtxRange nvtx("cusha_run");
  Graph& g = g0(h);
  const int a = (int)alg;
  const uint32_t V = h->st.num_vertices;
  if ((a == kBFS || a == kSSSP || a == kSSWP) && source >= V) return fail(CUSHA_EINVAL, "source >= num_vertices");
  if (alg_needs_edge_values(a) && !g.has_ev) return fail(CUSHA_EINVAL, "algorithm needs edge_values");
  if (alg_needs_init(a) && !g.d_init[a]) return fail(CUSHA_EINVAL, "NN/HS/CS need cusha_set_vertex_values first");
  const bool ranked = h->mode == kModeNccl || h->mode == kModeIpc;
  if (ranked && !g.connected) return fail(CUSHA_ESTATE, "the ranks are not connected yet (cusha_ipc_connect)");
  int rc = check_fixed_range(g, a);
  if (rc) return rc;
  CKA(cudaSetDevice(h->device));
  cudaStream_t st = h->stream;
  // trace buffer per partition, sized to min(max_iters, 2^20)
  const uint32_t want_cap = std::min<uint32_t>(std::max<uint32_t>(max_iters, 1), 1u << 20);
  for (Graph* p : h->parts) {
    if (p->trace_cap >= want_cap) continue;
    if (p->d_trace) cudaFreeAsync(p->d_trace, st);
    p->d_trace = nullptr;
    p->trace_cap = 0;
    CKA(dev_alloc((void**)&p->d_trace, sizeof(TraceRec) * (size_t)want_cap, st));
    CKA(cudaMemsetAsync(p->d_trace, 0, sizeof(TraceRec) * (size_t)want_cap, st));
    p->trace_cap = want_cap;
    p->trace_dirty = 0;
    for (auto& e : h->exec)  // kernel params captured the old trace pointer
      if (e) { cudaGraphExecDestroy(e); e = nullptr; }
    for (auto& e : h->chunk_exec)
      if (e) { cudaGraphExecDestroy(e); e = nullptr; }
  }
  const PassKernel& pk = pass_kernel(a, g.repr);
  if (!h->cfg_ok[a]) {
    if ((rc = pass_config(g, pk, &h->cfg[a]))) return rc;
    h->cfg_ok[a] = true;
  }
  const PassCfg& cfg = h->cfg[a];
  if (CUSHA_BIG_FIRST)
    for (Graph* p : h->parts)
      if (!pass_ahead(*p, a) && (rc = shard_order(*p))) return rc;
  for (Graph* p : h->parts)
    if ((rc = init_chunks(*p))) return rc;
  const bool parted = h->mode != kModeSingle;
  const bool host_loop = g.host_loop || parted || g.bsp;
  // one launch for the whole run (overlapped passes) unless asked otherwise;
  // the automatic mode takes one launch per pass for many small shards per
  // CTA (67_16 at |N| = 1536: 4.40 vs 5.48 ms)
  bool barrier = g.pass_barrier == 1;
  if (g.pass_barrier == 0 && g.S) {
    const uint64_t grid = pass_grid(g, pk, cfg.smem);
    barrier = (uint64_t)g.S >= 16 * grid && g.P <= 16384ull * g.S;
  }
  const bool multi = !host_loop && !barrier && max_iters <= g.trace_cap;
  if (!host_loop && !multi && (rc = ensure_exec(h, a, pk, cfg))) return rc;
  // records a previous run may have written (the rest are still zero)
  for (Graph* p : h->parts) {
    if (p->trace_dirty) CKA(cudaMemsetAsync(p->d_trace, 0, sizeof(TraceRec) * (size_t)p->trace_dirty, st));
    p->trace_dirty = p->trace_cap;  // until this run's extent is known
  }
  cudaEvent_t ev0 = g.ev0, evm = g.evm, ev1 = g.ev1;
  std::string err;
  CKA(cudaEventRecord(ev0, st));
  for (Graph* p : h->parts) CKA(launch_reset_ctl(p->d_ctl, max_iters, st));
  for (Graph* p : h->parts) CKA(launch_init(*p, a, source, st));
  // every partition's SrcValue is initialised (R20) before any pass reads it
  if (ranked) CKA(launch_peer_barrier(g, 0, g.comm_timeout_ms, st));
  CKA(cudaEventRecord(evm, st));
  if (max_iters > 0 && multi) {
    KParams kp = pass_params(g, source, cfg, a);
    kp.multi = 1;
    // passes in flight: 4 on low-degree graphs (road meshes need about their
    // diameter in passes, so the 2 extra confirming passes are amortised and
    // the wider overlap shortens each pass: C3 -6%), else 2 (power-law graphs
    // converge in a few passes, where the confirming passes would dominate;
    // DESIGN.md "Overlapped passes")
    kp.window = g.E < (uint64_t)kLowDegree * g.V ? kWideWindow : 2u;
    void* args[] = {&kp};
    CKA(cudaLaunchKernel(pk.func, dim3(cfg.grid), dim3(pk.threads), args, cfg.smem, st));
  } else if (max_iters > 0) {
    // passes in chunks; a pass that finds the run converged (or at max_iters)
    // exits at once, so over-launching is exact.  Partitioned: every
    // partition's pass, then the global convergence decision; every rank
    // takes it from the same all-reduced word, so all issue the same collectives.
    std::vector<KParams> kps;
    std::vector<uint32_t> grids;
    for (Graph* p : h->parts) {
      kps.push_back(pass_params(*p, source, cfg, a));
      grids.push_back(pass_grid(*p, pk, cfg.smem));
    }
    // one chunk = kChunk rounds of (every partition's pass [+ BSP copy], the
    // convergence decision); 16 passes per host check.  BSP alternates the two
    // SrcValue copies, an even number of times per chunk, so every chunk starts
    // from d_srcvalue.
    auto enqueue_chunk = [&](std::string& e2) -> int {
      uint32_t* cur = g.d_srcvalue;  // BSP: the copy this pass reads (init wrote d_srcvalue)
      uint32_t* nxt = g.d_srcvalue2;
      for (int k = 0; k < kChunk; ++k) {
        if (g.bsp) {
          // two-phase BSP: stage 4 writes the copy the NEXT pass reads, which
          // starts as this pass's input (entries no shard writes carry over)
          CKA(cudaMemcpyAsync(nxt, cur, 4 * (g.P + 1), cudaMemcpyDeviceToDevice, st));
          kps[0].srcvalue = cur;
          kps[0].sv_write = nxt;
          std::swap(cur, nxt);
        }
        for (size_t r = 0; r < h->parts.size(); ++r) {
          void* args[] = {&kps[r]};
          CKA(cudaLaunchKernel(pk.func, dim3(grids[r]), dim3(pk.threads), args, cfg.smem, st));
        }
        if (h->mode == kModeSim) {
          CKA(launch_close_parts(h->d_ctls, (uint32_t)h->parts.size(), st));
        } else if (ranked) {  // the barrier between ranks decides global convergence
          CKA(launch_peer_barrier(g, 1, g.comm_timeout_ms, st));
        }
        (void)e2;
      }
      return CUSHA_OK;
    };
    // partitioned / BSP chunks are captured once into a CUDA graph and replayed
    // (one launch per 16 rounds instead of (partitions + 2) x 16 API calls);
    // explicit host_loop (profilers) keeps the individual launches
    const bool capture = host_loop && !g.host_loop && !h->chunk_uncapturable[a];
    if (capture && !h->chunk_exec[a]) {
      cudaGraph_t cg = nullptr;
      bool ok = cudaStreamBeginCapture(st, cudaStreamCaptureModeThreadLocal) == cudaSuccess;
      std::string e2;
      const int crc = ok ? enqueue_chunk(e2) : CUSHA_OK;
      const cudaError_t ee = ok ? cudaStreamEndCapture(st, &cg) : cudaErrorUnknown;
      ok = ok && crc == CUSHA_OK && ee == cudaSuccess && cg;
      if (ok) ok = cudaGraphInstantiate(&h->chunk_exec[a], cg, 0) == cudaSuccess;
      if (cg) cudaGraphDestroy(cg);
      if (!ok) {  // run uncaptured (e.g. a library NCCL without stream-capture support)
        cudaGetLastError();
        h->chunk_exec[a] = nullptr;
        h->chunk_uncapturable[a] = true;
      }
    }
    for (;;) {
      if (host_loop) {
        if (h->chunk_exec[a]) {
          CKA(cudaGraphLaunch(h->chunk_exec[a], st));
        } else if ((rc = enqueue_chunk(err))) {
          return rc;
        }
      } else {
        CKA(cudaGraphLaunch(h->exec[a], st));
      }
      CKA(cudaMemcpyAsync(g.h_ctl, g.d_ctl, sizeof(Ctl), cudaMemcpyDeviceToHost, st));
      CKA(cudaStreamSynchronize(st));  // (the barrier between ranks is bounded by comm_timeout_ms)
      if (ranked) {
        uint32_t perr = 0;
        CKA(cudaMemcpy(&perr, &g.d_sync->err, 4, cudaMemcpyDeviceToHost));
        if (perr) return fail(CUSHA_ENCCL, "a rank did not reach the pass barrier within comm_timeout_ms");
      }
      if (g.h_ctl->converged || g.h_ctl->iter >= max_iters) break;
    }
  }
  CKA(cudaEventRecord(ev1, st));
  // one round trip for every partition's Ctl block and the head of its trace
  // (the rest, for runs longer than kHostTrace passes, in read_trace)
  for (Graph* p : h->parts) {
    CKA(cudaMemcpyAsync(p->h_ctl, p->d_ctl, sizeof(Ctl), cudaMemcpyDeviceToHost, st));
    const uint32_t nt = std::min(kHostTrace, p->trace_cap);
    if (nt) CKA(cudaMemcpyAsync(p->h_trace, p->d_trace, sizeof(TraceRec) * nt, cudaMemcpyDeviceToHost, st));
  }
  CKA(cudaStreamSynchronize(st));
  float ms = 0, lms = 0;
  cudaEventElapsedTime(&ms, ev0, ev1);
  cudaEventElapsedTime(&lms, evm, ev1);
  // statistics and algorithmic bytes, per partition and summed
  cusha_stats sum{};
  Ctl c0{};
  for (size_t r = 0; r < h->parts.size(); ++r) {
    Graph& p = *h->parts[r];
    Ctl c = *p.h_ctl;
    {  // passes whose trace records this run touched: its iterations, or every drawn ticket's pass
      const uint64_t drawn = multi && p.Sl ? c.ticket / p.Sl + 1 : 0;
      p.trace_dirty = (uint32_t)std::min<uint64_t>(p.trace_cap, std::max<uint64_t>(c.iter, drawn) + 2);
    }
    if (multi && max_iters > 0) {  // the confirming pass that committed nothing, else max_iters passes ran
      c.converged = c.conv_iter != 0xFFFFFFFFu;
      c.iter = c.converged ? c.conv_iter : max_iters;
    }
    std::vector<TraceRec> tr;
    const uint32_t ntr = std::min(c.iter, p.trace_cap);
    if (ntr <= kHostTrace) tr.assign(p.h_trace, p.h_trace + std::max<uint32_t>(ntr, 1));
    else if ((rc = read_trace(p, ntr, tr))) return rc;
    account_run(p, a, c, multi, cfg.mapj != 0, p.st, tr);
    p.st.run_ms = ms;
    p.st.loop_ms = lms;
    if (r == 0) c0 = c;
    sum.algorithmic_bytes += p.st.algorithmic_bytes;
    sum.paper_bytes += p.st.paper_bytes;
    sum.edges_processed += p.st.edges_processed;
    sum.wb_entries += p.st.wb_entries;
    sum.vertices_processed += p.st.vertices_processed;
    sum.updated_total += p.st.updated_total;
    sum.stage2_bytes_per_iter += p.st.stage2_bytes_per_iter;
    sum.wb_bytes_all_active += p.st.wb_bytes_all_active;
  }
  cusha_stats& s = h->st;
  s.iterations = c0.iter;
  s.converged = c0.converged;
  s.run_ms = ms;
  s.loop_ms = lms;
  s.last_algorithm = a;
  s.algorithmic_bytes = sum.algorithmic_bytes;
  s.paper_bytes = sum.paper_bytes;
  s.edges_processed = sum.edges_processed;
  s.wb_entries = sum.wb_entries;
  s.vertices_processed = sum.vertices_processed;
  s.updated_total = sum.updated_total;
  s.stage2_bytes_per_iter = sum.stage2_bytes_per_iter;
  s.wb_bytes_all_active = sum.wb_bytes_all_active;
  s.mapper_form = (uint32_t)cfg.mapj;
  s.ring_slots = cfg.nst;
  s.l2_read_ahead = (uint32_t)pass_ahead(g, a);
  s.device_loop = host_loop ? 0 : (multi ? 2 : 1);
  h->last_alg = a;
  h->have_values = true;
  return c0.converged ? CUSHA_OK : CUSHA_NOT_CONVERGED;
}

// copy every partition's VertexValues slice to dst (host or device)
static int copy_values(const cusha_graph* h, void* dst, bool to_host) {
  const size_t vb = value_bytes(h->last_alg);
  const cudaMemcpyKind kind = to_host ? cudaMemcpyDeviceToHost : cudaMemcpyDeviceToDevice;
  if (h->mode == kModeNccl || h->mode == kModeIpc) {
    // every rank reads every rank's slice from its memory (CUDA IPC): a
    // barrier before (all ranks finished their runs) and after (no rank frees
    // or overwrites its slice while another still reads it); collective
    Graph& g = *h->parts[0];
    CKA(launch_peer_barrier(g, 0, g.comm_timeout_ms, h->stream));
    for (uint32_t q = 0; q < g.G; ++q) {
      const uint64_t v0 = std::min<uint64_t>((uint64_t)g.h_bounds[q] * g.N, g.V);
      const uint64_t v1 = std::min<uint64_t>((uint64_t)g.h_bounds[q + 1] * g.N, g.V);
      if (v1 > v0)
        CKA(cudaMemcpyAsync(static_cast<char*>(dst) + v0 * vb, g.vv_peer[q], (v1 - v0) * vb,
                            to_host ? cudaMemcpyDeviceToHost : cudaMemcpyDefault, h->stream));
    }
    CKA(launch_peer_barrier(g, 0, g.comm_timeout_ms, h->stream));
    CKA(cudaStreamSynchronize(h->stream));
    uint32_t perr = 0;
    CKA(cudaMemcpy(&perr, &g.d_sync->err, 4, cudaMemcpyDeviceToHost));
    if (perr) return fail(CUSHA_ENCCL, "a rank did not reach the barrier within comm_timeout_ms");
    return CUSHA_OK;
  }
  for (const Graph* g : h->parts)
    if (g->nvl)
      CKA(cudaMemcpyAsync(static_cast<char*>(dst) + (size_t)g->v0 * vb, g->d_vv, (size_t)g->nvl * vb, kind,
                          h->stream));
  CKA(cudaStreamSynchronize(h->stream));
  return CUSHA_OK;
}

int cusha_get_values(const cusha_graph* h, void* out, size_t out_bytes) {
  if (!h || !out) return fail(CUSHA_EINVAL, "null argument");
  if (!h->have_values) return fail(CUSHA_ESTATE, "no run yet");
  const size_t want = (size_t)h->st.num_vertices * value_bytes(h->last_alg);
  if (out_bytes != want) return fail(CUSHA_EINVAL, "out_bytes must be |V| * value_bytes(last algorithm)");
  NvtxRange nvtx("cusha_get_values");
  CKA(cudaSetDevice(h->device));
  return copy_values(h, out, true);
}

int cusha_get_values_device(const cusha_graph* h, void* dptr, size_t out_bytes) {
  if (!h || !dptr) return fail(CUSHA_EINVAL, "null argument");
  if (!h->have_values) return fail(CUSHA_ESTATE, "no run yet");
  const size_t want = (size_t)h->st.num_vertices * value_bytes(h->last_alg);
  if (out_bytes != want) return fail(CUSHA_EINVAL, "out_bytes must be |V| * value_bytes(last algorithm)");
  CKA(cudaSetDevice(h->device));
  return copy_values(h, dptr, false);
}

int cusha_get_stats(const cusha_graph* h, cusha_stats* s) {
  if (!h || !s) return fail(CUSHA_EINVAL, "null argument");
  *s = h->st;
  return CUSHA_OK;
}

int cusha_get_part_stats(const cusha_graph* h, uint32_t part, cusha_stats* s) {
  if (!h || !s) return fail(CUSHA_EINVAL, "null argument");
  if (part >= h->parts.size()) return fail(CUSHA_EINVAL, "partition not held by this handle");
  const Graph& g = *h->parts[part];
  *s = h->st;
  s->device_bytes = device_bytes(g);
  s->max_part_device_bytes = s->device_bytes;
  s->entries_padded = g.P;
  s->rank = (h->mode == kModeNccl || h->mode == kModeIpc) ? h->st.rank : (int)part;
  if (h->have_values) {
    s->algorithmic_bytes = g.st.algorithmic_bytes;
    s->paper_bytes = g.st.paper_bytes;
    s->edges_processed = g.st.edges_processed;
    s->wb_entries = g.st.wb_entries;
    s->vertices_processed = g.st.vertices_processed;
    s->updated_total = g.st.updated_total;
    s->stage2_bytes_per_iter = g.st.stage2_bytes_per_iter;
    s->wb_bytes_all_active = g.st.wb_bytes_all_active;
  }
  return CUSHA_OK;
}

int cusha_get_trace(const cusha_graph* h, uint32_t* upd, uint32_t* act, uint32_t cap) {
  if (!h) return fail(CUSHA_EINVAL, "null argument");
  if (!h->have_values) return 0;
  const uint32_t n = std::min(std::min(h->st.iterations, g0(h).trace_cap), cap);
  if (!n) return 0;
  cudaSetDevice(h->device);
  std::vector<uint64_t> su(n, 0), sa(n, 0);
  for (const Graph* g : h->parts) {  // summed over the partitions of this handle
    std::vector<TraceRec> tr;
    const int rc = read_trace(*g, n, tr);
    if (rc) return rc;
    for (uint32_t i = 0; i < n; ++i) {
      su[i] += tr[i].updated;
      sa[i] += tr[i].active_shards;
    }
  }
  for (uint32_t i = 0; i < n; ++i) {
    if (upd) upd[i] = (uint32_t)su[i];
    if (act) act[i] = (uint32_t)sa[i];
  }
  return (int)n;
}

static int layout_of(const Graph& g, cusha_layout_part part, void* out, size_t out_bytes, uint64_t* count) {
  const void* src = nullptr;
  const void* tail = nullptr;  // host-resident part (row f3) from position `split`
  uint64_t n = 0, split = ~0ull;
  size_t es = 4;
  switch (part) {
    case CUSHA_LAYOUT_SHARD_OFFSETS: src = g.d_shard_off; n = (uint64_t)g.Sl + 1; break;
    case CUSHA_LAYOUT_SHARD_SIZES: src = g.d_shard_cnt; n = g.Sl; break;
    case CUSHA_LAYOUT_SRC_INDEX: src = g.d_srcloc; tail = g.h_srcloc; split = g.splitP; n = g.P; es = 2; break;
    case CUSHA_LAYOUT_DEST_LOCAL: src = g.d_dest; tail = g.h_dest; split = g.splitP; n = g.P; es = 2; break;
    case CUSHA_LAYOUT_EDGE_ID: src = g.d_eid; tail = g.h_eid; split = g.splitP; n = g.P; break;
    case CUSHA_LAYOUT_WINDOWS: src = g.d_win; n = ((uint64_t)g.Sl + 1) * g.S; break;
    case CUSHA_LAYOUT_CW_OFFSETS: src = g.d_cw_off; n = (uint64_t)g.Sl + 1; break;
    case CUSHA_LAYOUT_CW_SIZES: src = g.d_cw_cnt; n = g.Sl; break;
    case CUSHA_LAYOUT_CW_SRC_LOCAL: src = g.d_cw_src; tail = g.h_cw_src; split = g.splitQ; n = g.Q; es = 2; break;
    case CUSHA_LAYOUT_MAPPER: src = g.d_mapper; tail = g.h_mapper; split = g.splitQ; n = g.Q; break;
    case CUSHA_LAYOUT_OUT_DEGREE: src = g.d_outdeg; n = g.nvl; break;
    case CUSHA_LAYOUT_RUN_K: src = g.d_run_k; n = g.R; break;
    case CUSHA_LAYOUT_RUN_T: src = g.d_run_t; n = g.R; break;
    case CUSHA_LAYOUT_CW_WINDOW: src = g.d_cw_win; tail = g.h_cw_win; split = g.splitQ; n = g.Q; es = 2; break;
    case CUSHA_LAYOUT_CW_DELTA: src = g.d_cw_delta; n = (uint64_t)g.Sl * g.S; break;
    case CUSHA_LAYOUT_CW_PARTITION_OFFSETS: src = g.d_cwp; n = (uint64_t)g.Sl * (g.G + 1); break;
    default: return fail(CUSHA_EINVAL, "bad layout part");
  }
  if (!src && !tail) return fail(CUSHA_EUNSUPPORTED, "part not held by this graph (representation / options)");
  if (count) *count = n;
  if (!out) return CUSHA_OK;
  if (out_bytes < n * es) return fail(CUSHA_EINVAL, "out_bytes too small");
  CKA(cudaSetDevice(g.device));
  const uint64_t nd = std::min(n, split);  // HBM part
  if (nd) {
    CKA(cudaMemcpyAsync(out, src, nd * es, cudaMemcpyDeviceToHost, g.stream));
    CKA(cudaStreamSynchronize(g.stream));
  }
  if (nd < n) std::memcpy(static_cast<char*>(out) + nd * es, tail, (n - nd) * es);
  return CUSHA_OK;
}

int cusha_get_layout(const cusha_graph* h, cusha_layout_part part, void* out, size_t out_bytes, uint64_t* count) {
  if (!h) return fail(CUSHA_EINVAL, "graph is NULL");
  if (h->mode != kModeSingle)
    return fail(CUSHA_EUNSUPPORTED, "partitioned graph: use cusha_get_part_layout");
  return layout_of(g0(h), part, out, out_bytes, count);
}

int cusha_get_part_layout(const cusha_graph* h, uint32_t p, cusha_layout_part part, void* out, size_t out_bytes,
                          uint64_t* count) {
  if (!h) return fail(CUSHA_EINVAL, "graph is NULL");
  if (p >= h->parts.size()) return fail(CUSHA_EINVAL, "partition not held by this handle");
  return layout_of(*h->parts[p], part, out, out_bytes, count);
}

int cusha_ipc_export(cusha_graph* h, void* out, size_t bytes) {
  if (!h || !out) return fail(CUSHA_EINVAL, "null argument");
  if (h->mode != kModeIpc && h->mode != kModeNccl) return fail(CUSHA_ESTATE, "not a one-process-per-GPU graph");
  if (bytes != kIpcBlob) return fail(CUSHA_EINVAL, "bytes must be CUSHA_IPC_BLOB_BYTES");
  CKA(cudaSetDevice(h->device));
  return ipc_export_blob(*h->parts[0], out);
}

int cusha_ipc_connect(cusha_graph* h, const void* all, size_t bytes) {
  if (!h || !all) return fail(CUSHA_EINVAL, "null argument");
  if (h->mode != kModeIpc) return fail(CUSHA_ESTATE, "not a caller-bootstrapped (transport IPC) graph");
  Graph& g = *h->parts[0];
  if (g.connected) return fail(CUSHA_ESTATE, "already connected");
  if (bytes != kIpcBlob * g.G) return fail(CUSHA_EINVAL, "bytes must be world_size * CUSHA_IPC_BLOB_BYTES");
  CKA(cudaSetDevice(h->device));
  return ipc_connect_blob(g, all);
}

int cusha_nccl_unique_id(void* out128) {
  if (!out128) return fail(CUSHA_EINVAL, "out128 is NULL");
  std::string err;
  const int rc = nccl_unique_id(out128, err);
  return rc ? fail(rc, err) : CUSHA_OK;
}

int cusha_partition_shards(uint32_t num_shards, const uint64_t* work, uint32_t parts, uint32_t* bounds) {
  if (!work || !bounds || parts == 0) return fail(CUSHA_EINVAL, "null argument or parts == 0");
  partition_bounds(num_shards, work, parts, bounds);
  return CUSHA_OK;
}

int cusha_get_partition(const cusha_graph* h, uint32_t* bounds, uint32_t cap) {
  if (!h || !bounds) return fail(CUSHA_EINVAL, "null argument");
  const std::vector<uint32_t>& b = g0(h).h_bounds;
  const uint32_t G = (uint32_t)b.size() - 1;
  if (cap < G + 1) return fail(CUSHA_EINVAL, "cap too small");
  for (uint32_t q = 0; q <= G; ++q) bounds[q] = b[q];
  return (int)G;
}

int cusha_diag_timeline(void* out, size_t out_bytes) {
  if (!out) return fail(CUSHA_EINVAL, "null argument");
  cudaDeviceSynchronize();
  const int n = timeline_copy(out, out_bytes);
  return n < 0 ? fail(CUSHA_EUNSUPPORTED, "library built without CUSHA_TIMELINE") : n;
}

}  // extern "C"
