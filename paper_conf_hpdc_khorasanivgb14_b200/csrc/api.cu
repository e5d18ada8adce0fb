// api.cu — the C ABI of include/cusha.h (row b) and the iteration driver (row a5).
//
// cusha_run replaces the paper's host loop (Fig. 5 lines 0-2 and 29; L189:
// launch, cudaMemcpy(is_converged), decide) by ONE launch of a CUDA graph
// whose body is the shard pass under a conditional while node; the shard
// pass's last CTA decides whether the loop goes on (DESIGN.md "Iteration
// control").  The host waits once, at the end.
#include <algorithm>
#include <chrono>
#include <cmath>
#include <cstring>
#include <string>

#include "algorithms.cuh"
#include "graph.hpp"

struct cusha_graph {
  cusha::Graph g;
  cudaGraphExec_t exec[cusha::kNumAlgs] = {};
  bool exec_failed[cusha::kNumAlgs] = {};
};

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

static void free_graph_memory(Graph& g) {
  void* ptrs[] = {g.d_shard_off, g.d_shard_cnt, g.d_dest, g.d_srcloc, g.d_eid, g.d_ev, g.d_win, g.d_cw_off,
                  g.d_cw_cnt, g.d_cw_src, g.d_mapper, g.d_outdeg, g.d_srcvalue, g.d_vv, g.d_ctl, g.d_trace,
                  g.d_active, g.d_bounds, g.d_owner, g.d_cwp, g.d_gathered, g.d_run_k, g.d_run_t,
                  g.d_run_unit, g.d_run_bits, g.d_run_d, g.d_dirty, g.d_shard_seq, g.d_cw_win, g.d_cw_delta};
  nccl_destroy(g);
  // device memory is stream-ordered (cudaMallocAsync on g.stream): released to
  // the retained pool without unmapping or a device-wide synchronisation
  for (void* p : ptrs)
    if (p) cudaFreeAsync(p, g.stream);
  for (void*& p : g.d_init)
    if (p) { cudaFreeAsync(p, g.stream); p = nullptr; }
  void* hosts[] = {g.h_dest, g.h_ev, g.h_srcloc, g.h_eid, g.h_cw_src, g.h_mapper, g.h_cw_win};
  for (void* p : hosts)
    if (p) cudaFreeHost(p);
  delete g.h_ctl;
  g.h_ctl = nullptr;
  if (g.ev0) cudaEventDestroy(g.ev0);
  if (g.ev1) cudaEventDestroy(g.ev1);
  if (g.evm) cudaEventDestroy(g.evm);
  if (g.own_stream && g.stream) {
    cudaStreamSynchronize(g.stream);
    cudaStreamDestroy(g.stream);
  }
}

// Keep freed device memory in the default pool so that repeated builds (the
// e2e path) reuse it instead of mapping HBM again.
static void retain_pool(int device) {
  cudaMemPool_t pool;
  if (cudaDeviceGetDefaultMemPool(&pool, device) == cudaSuccess) {
    uint64_t keep = UINT64_MAX;
    cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &keep);
  }
}

static uint64_t device_bytes(const Graph& g) {
  uint64_t b = 4ull * (g.S + 1) * 2 + 4ull * g.S * 2;  // offsets + counts
  b += 2 * g.P + 4 * g.P;                               // dest + eid
  if (g.has_ev) b += 4 * g.P;
  if (g.d_srcloc) b += 2 * g.P;
  if (g.d_win) b += 4ull * (g.S + 1) * g.S;
  b += (2 + 4 + 2) * g.Q;                               // CW: SrcIndexCW, Mapper, window
  if (g.d_cw_delta) b += 4ull * g.S * g.S;             // Mapper deltas per window
  b += 4ull * g.V;                                      // outdeg
  b += 4 * (g.P + 1) + 8ull * g.V;                      // SrcValue + VertexValues
  return b - g.host_bytes;                              // minus the host-streamed part (row f3)
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
  if (o.world_size > 1 && o.nccl_unique_id && (o.rank < 0 || o.rank >= o.world_size))
    return fail(CUSHA_EINVAL, "rank out of range");
  uint32_t N = o.vertices_per_shard ? o.vertices_per_shard : cusha_shard_size(V, E, o.smem_bytes_per_vertex, 0, 0);
  if (N > 65534) return fail(CUSHA_EINVAL, "vertices_per_shard must be <= 65534");
  if (o.pass_barrier < 0 || o.pass_barrier > 2) return fail(CUSHA_EINVAL, "pass_barrier must be 0, 1 or 2");
  if (N > V) N = V;

  cusha_graph* h = new (std::nothrow) cusha_graph();
  if (!h) return fail(CUSHA_ENOMEM, "host allocation");
  Graph& g = h->g;
  g.V = V; g.E = E; g.N = N; g.S = (V + N - 1) / N; g.repr = (int)o.repr; g.device = o.device;
  g.host_loop = o.host_loop != 0;
  g.skip_clean = o.skip_clean_shards != 0;
  g.pass_barrier = o.pass_barrier;
  g.topo_budget = o.device_topology_budget;
  g.world_size = o.world_size;
  g.rank = o.world_size > 1 && o.nccl_unique_id ? o.rank : 0;
  g.simulate = o.world_size > 1 && !o.nccl_unique_id;
  g.G = std::min<uint32_t>((uint32_t)o.world_size, g.S);  // never more partitions than shards
  if (!g.simulate && g.G != (uint32_t)o.world_size) {
    delete h;
    return fail(CUSHA_EINVAL, "world_size exceeds the number of shards");
  }
  auto bail = [&](int code) { free_graph_memory(g); delete h; return code; };
  auto cu = [&](cudaError_t e, const char* what) -> int {
    if (e == cudaSuccess) return 0;
    set_error(std::string(what) + ": " + cudaGetErrorString(e));
    return e == cudaErrorMemoryAllocation ? CUSHA_ENOMEM : CUSHA_ECUDA;
  };
  int rc;
  if ((rc = cu(cudaSetDevice(o.device), "cudaSetDevice"))) return bail(rc);
  retain_pool(o.device);
  if (o.stream) {
    g.stream = (cudaStream_t)o.stream;
  } else {
    if ((rc = cu(cudaStreamCreateWithFlags(&g.stream, cudaStreamNonBlocking), "cudaStreamCreate"))) return bail(rc);
    g.own_stream = true;
  }
  if ((rc = cu(cudaEventCreate(&g.ev0), "cudaEventCreate")) || (rc = cu(cudaEventCreate(&g.ev1), "cudaEventCreate")) ||
      (rc = cu(cudaEventCreate(&g.evm), "cudaEventCreate")))
    return bail(rc);
  cudaEvent_t eh = nullptr;
  if ((rc = cu(cudaEventCreate(&eh), "cudaEventCreate"))) return bail(rc);

  auto t0 = std::chrono::steady_clock::now();
  CKA(cudaEventRecord(g.ev0, g.stream));
  const uint32_t *d_src = src, *d_dst = dst, *d_val = edge_values;
  uint32_t* tmp = nullptr;
  uint64_t h2d = 0;
  if (o.input_location == CUSHA_INPUT_HOST && E) {
    const uint64_t nvals = edge_values ? 3 : 2;
    if ((rc = cu(cudaMallocAsync(&tmp, nvals * E * 4, g.stream), "cudaMallocAsync(inputs)"))) {
      cudaEventDestroy(eh);
      return bail(rc);
    }
    cudaMemcpyAsync(tmp, src, E * 4, cudaMemcpyHostToDevice, g.stream);
    cudaMemcpyAsync(tmp + E, dst, E * 4, cudaMemcpyHostToDevice, g.stream);
    if (edge_values) cudaMemcpyAsync(tmp + 2 * E, edge_values, E * 4, cudaMemcpyHostToDevice, g.stream);
    d_src = tmp; d_dst = tmp + E; d_val = edge_values ? tmp + 2 * E : nullptr;
    h2d = nvals * E * 4;
  }
  cudaEventRecord(eh, g.stream);
  std::string err;
  rc = build_layout(g, d_src, d_dst, d_val, err);
  if (rc) {
    if (tmp) cudaFreeAsync(tmp, g.stream);
    cudaEventDestroy(eh);
    set_error("build: " + err);
    return bail(rc);
  }
  if (tmp) cudaFreeAsync(tmp, g.stream);
  if (g.G > 1) {  // destination-range partition (row e)
    rc = build_partition(g, err);
    if (!rc && !g.simulate) rc = nccl_init(g, o.nccl_unique_id, err);
    if (rc) {
      cudaEventDestroy(eh);
      set_error("partition: " + err);
      return bail(rc);
    }
  }
  rc = offload_topology(g, err);  // row f3 (no-op without a budget)
  if (rc) {
    cudaEventDestroy(eh);
    set_error("host topology: " + err);
    return bail(rc);
  }
  // per-run state: SrcValue (P entries + trash slot), VertexValues (8 B/vertex covers every Table-3 Vertex)
  g.h_ctl = new (std::nothrow) Ctl();
  if ((rc = cu(cudaMallocAsync(&g.d_srcvalue, 4 * (g.P + 1), g.stream), "cudaMallocAsync(SrcValue)")) ||
      (rc = cu(cudaMemsetAsync(g.d_srcvalue, 0, 4 * (g.P + 1), g.stream), "memset")) ||
      (rc = cu(cudaMallocAsync(&g.d_vv, 8ull * V, g.stream), "cudaMallocAsync(VertexValues)")) ||
      (rc = cu(cudaMallocAsync(&g.d_ctl, sizeof(Ctl), g.stream), "cudaMallocAsync(ctl)")) ||
      (rc = g.h_ctl ? 0 : CUSHA_ENOMEM)) {
    cudaEventDestroy(eh);
    return bail(rc);
  }
  CKA(cudaEventRecord(g.ev1, g.stream));
  CKA(cudaEventSynchronize(g.ev1));
  float ms = 0, ms_h2d = 0;
  cudaEventElapsedTime(&ms, g.ev0, g.ev1);
  cudaEventElapsedTime(&ms_h2d, g.ev0, eh);
  cudaEventDestroy(eh);
  (void)t0;
  g.st.num_vertices = V;
  g.st.num_edges = E;
  g.st.vertices_per_shard = N;
  g.st.num_shards = g.S;
  g.st.repr = (uint32_t)g.repr;
  g.st.last_algorithm = -1;
  g.st.build_ms = ms;
  g.st.h2d_ms = ms_h2d;
  g.st.h2d_bytes = h2d;
  g.st.device_bytes = device_bytes(g);
  g.st.entries_padded = g.P;
  g.st.world_size = g.world_size;
  g.st.rank = g.rank;
  g.st.host_bytes = g.host_bytes;
  g.st.host_shard = g.host_shard;
  *out = h;
  set_error("");
  return CUSHA_OK;
}

void cusha_free_graph(cusha_graph* h) {
  if (!h) return;
  cudaSetDevice(h->g.device);
  for (auto& e : h->exec)
    if (e) cudaGraphExecDestroy(e);
  free_graph_memory(h->g);
  delete h;
}

int cusha_set_vertex_values(cusha_graph* h, cusha_algorithm alg, const void* init, size_t bytes) {
  if (!h || !init) return fail(CUSHA_EINVAL, "null argument");
  if ((int)alg < 0 || (int)alg >= kNumAlgs) return fail(CUSHA_EINVAL, "bad algorithm");
  Graph& g = h->g;
  const size_t want = (size_t)g.V * value_bytes((int)alg);
  if (bytes != want) return fail(CUSHA_EINVAL, "bytes must be |V| * value_bytes(alg)");
  CKA(cudaSetDevice(g.device));
  if (!g.d_init[alg]) CKA(cudaMallocAsync(&g.d_init[alg], want, g.stream));
  CKA(cudaMemcpyAsync(g.d_init[alg], init, want, cudaMemcpyHostToDevice, g.stream));
  CKA(cudaStreamSynchronize(g.stream));
  return CUSHA_OK;
}

// Persistent grid of the shard pass: as many CTAs as fit on the device at
// once (occupancy x SMs), never more than there are shards.
static uint32_t pass_grid(const Graph& g, const PassKernel& pk, size_t smem) {
  // shards this process runs: its partition (multi-GPU) or all of them
  const uint32_t mine = g.G > 1 && !g.simulate ? g.h_bounds[g.rank + 1] - g.h_bounds[g.rank] : g.S;
  if (!pk.persistent) return std::max<uint32_t>(mine, 1);
  int sms = 148, per_sm = 1;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, g.device);
  if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, pk.func, (int)pk.threads, smem) != cudaSuccess ||
      per_sm < 1)
    per_sm = 1;
  const uint64_t gsz = (uint64_t)sms * (uint64_t)per_sm;
  return (uint32_t)std::max<uint64_t>(1, std::min<uint64_t>(gsz, mine));
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
#ifndef CUSHA_STASH
#define CUSHA_STASH 1  // 0: stage 3 of the integer algorithms re-reads VertexValues (tuning comparison)
#endif
static int pass_config(const Graph& g, const PassKernel& pk, size_t* smem, int* mapj, int* stash, uint32_t* nst) {
  cudaFuncAttributes fa{};
  CKA(cudaFuncGetAttributes(&fa, pk.func));
  const size_t kMaxSmem = 227 * 1024 - fa.sharedSizeBytes;  // dynamic part of the 227 KB per-CTA limit
  const size_t sm_m = pk.smem_bytes(g.N);
  if (sm_m > kMaxSmem)
    return fail(CUSHA_EINVAL, "vertices_per_shard too large for this algorithm's shared-memory state");
  CKA(cudaFuncSetAttribute(pk.func, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kMaxSmem));
  CKA(cudaFuncSetAttribute(pk.func, cudaFuncAttributePreferredSharedMemoryCarveout, cudaSharedmemCarveoutMaxShared));
  *smem = sm_m;
  *mapj = 0;
  const size_t sm_j = pk.smem_bytes(g.N, g.S);
  // ... and only when the rows cost less traffic than they save: an active
  // shard reads its 4|S|-byte row, so |S| rows per pass (4|S|^2 bytes) against
  // 2 bytes per CW entry (|Q| entries) saved over the u32 Mapper
  const bool row_pays = 4ull * g.S * g.S <= (uint64_t)g.Q;
  if (CUSHA_MAPJ && row_pays && g.repr == CUSHA_REPR_CW && g.d_cw_win && g.d_cw_delta && !kernels_rle() &&
      g.S <= 0xFFFFu && sm_j <= kMaxSmem) {
    int occ_m = 0, occ_j = 0;
    CKA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ_m, pk.func, (int)pk.threads, sm_m));
    CKA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ_j, pk.func, (int)pk.threads, sm_j));
    if (occ_j >= occ_m && occ_j > 0) {
      *smem = sm_j;
      *mapj = 1;
    }
  }
  // integer algorithms: keep the shard's VertexValues from stage 1 in shared
  // memory for stage 3's update_condition (no second global read) whenever
  // that costs no CTAs per SM
  *stash = 0;
  const size_t sm_s = *smem + 4ull * g.N;
  if (CUSHA_STASH && pk.monotone && sm_s <= kMaxSmem) {
    int occ_0 = 0, occ_s = 0;
    CKA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ_0, pk.func, (int)pk.threads, *smem));
    CKA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ_s, pk.func, (int)pk.threads, sm_s));
    if (occ_s >= occ_0 && occ_s > 0) {
      *smem = sm_s;
      *stash = 1;
    }
  }
  // a deeper TMA ring whenever another slot fits at the same CTAs per SM
  // (more bytes in flight per SM; e.g. C5 at one CTA per SM)
  *nst = pk.ring_bytes / pk.slot_bytes;
  if (CUSHA_DEEP_RING) {
    int occ_0 = 0;
    CKA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ_0, pk.func, (int)pk.threads, *smem));
    while (*nst < pk.max_stages && *smem + pk.slot_bytes <= kMaxSmem) {
      int occ_d = 0;
      CKA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ_d, pk.func, (int)pk.threads, *smem + pk.slot_bytes));
      if (occ_d < occ_0 || occ_d == 0) break;
      *smem += pk.slot_bytes;
      ++*nst;
    }
  }
  return CUSHA_OK;
}

// L2 prefetch of stage-2 tiles beyond the ring (KParams::ahead) pays when a
// pass streams from HBM; on passes that stay in L2 it only adds producer
// latency: on when the entry streams of one pass
// exceed twice the L2.
static int pass_ahead(const Graph& g, int alg) {
  int l2 = 0;
  if (cudaDeviceGetAttribute(&l2, cudaDevAttrL2CacheSize, g.device) != cudaSuccess || l2 <= 0) l2 = 126 << 20;
  const uint64_t bytes = (uint64_t)g.P * (6 + (alg_needs_edge_values(alg) ? 4 : 0)) + (uint64_t)g.Q * 8;
  return bytes > 2ull * (uint64_t)l2 ? 1 : 0;
}

#ifndef CUSHA_DIAG_FIXED_GRAPH
#define CUSHA_DIAG_FIXED_GRAPH 0
#endif
#ifndef CUSHA_DIAG_COND_NODE
#define CUSHA_DIAG_COND_NODE 0
#endif
#if CUSHA_DIAG_COND_NODE
// sanitizer diagnostic only: the while condition set by a one-thread kernel
// after the pass (the pass runs with use_cond = 0 and closes the iteration)
__global__ void diag_set_cond(const Ctl* ctl, cudaGraphConditionalHandle h) {
  const uint32_t more = !*reinterpret_cast<const volatile uint32_t*>(&ctl->converged) && ctl->iter < ctl->max_iters;
  cudaGraphSetConditional(h, more ? 1u : 0u);
}
#endif
static int ensure_exec(cusha_graph* h, int alg) {
  Graph& g = h->g;
  if (h->exec[alg]) return CUSHA_OK;
  const PassKernel& pk = pass_kernel(alg, g.repr);
  size_t smem = 0;
  int mapj = 0, stash = 0;
  uint32_t nst = 0;
  const int prc = pass_config(g, pk, &smem, &mapj, &stash, &nst);
  if (prc) return prc;
  cudaGraph_t graph = nullptr;
  CKA(cudaGraphCreate(&graph, 0));
#if CUSHA_DIAG_FIXED_GRAPH
  // sanitizer diagnostic only (profiles/r1/sanitizer/README.md): a chain of
  // CUSHA_DIAG_FIXED_GRAPH per-pass launches without the conditional node; a
  // pass launched after convergence is a no-op, as in the host loop
  {
    KParams kp = make_params(g, 0);
    kp.mapj = mapj;
    kp.stash = stash;
    kp.nst = nst;
    kp.ahead = pass_ahead(g, alg);
    void* args[] = {&kp};
    cudaKernelNodeParams knp = {};
    knp.func = const_cast<void*>(pk.func);
    knp.gridDim = dim3(pass_grid(g, pk, smem));
    knp.blockDim = dim3(pk.threads);
    knp.sharedMemBytes = (unsigned)smem;
    knp.kernelParams = args;
    cudaGraphNode_t prev = nullptr, kn;
    cudaError_t e = cudaSuccess;
    for (int i = 0; i < CUSHA_DIAG_FIXED_GRAPH && e == cudaSuccess; ++i) {
      e = cudaGraphAddKernelNode(&kn, graph, prev ? &prev : nullptr, prev ? 1 : 0, &knp);
      prev = kn;
    }
    if (e == cudaSuccess) e = cudaGraphInstantiate(&h->exec[alg], graph, 0);
    cudaGraphDestroy(graph);
    if (e != cudaSuccess) { h->exec[alg] = nullptr; return fail(CUSHA_ECUDA, std::string("graph: ") + cudaGetErrorString(e)); }
    return CUSHA_OK;
  }
#endif
  cudaGraphConditionalHandle handle;
  cudaError_t e = cudaGraphConditionalHandleCreate(&handle, graph, 1, cudaGraphCondAssignDefault);
  if (e != cudaSuccess) { cudaGraphDestroy(graph); return fail(CUSHA_ECUDA, std::string("conditional handle: ") + cudaGetErrorString(e)); }
  cudaGraphNodeParams cp = {};
  cp.type = cudaGraphNodeTypeConditional;
  cp.conditional.handle = handle;
  cp.conditional.type = cudaGraphCondTypeWhile;
  cp.conditional.size = 1;
  cudaGraphNode_t cnode;
  e = cudaGraphAddNode(&cnode, graph, nullptr, 0, &cp);
  if (e != cudaSuccess) { cudaGraphDestroy(graph); return fail(CUSHA_ECUDA, std::string("conditional node: ") + cudaGetErrorString(e)); }
  cudaGraph_t body = cp.conditional.phGraph_out[0];
  KParams kp = make_params(g, 0);
  kp.use_cond = CUSHA_DIAG_COND_NODE ? 0 : 1;
  kp.mapj = mapj;
  kp.stash = stash;
  kp.nst = nst;
  kp.ahead = pass_ahead(g, alg);
  kp.cond_handle = handle;
  void* args[] = {&kp};
  cudaKernelNodeParams knp = {};
  knp.func = const_cast<void*>(pk.func);
  knp.gridDim = dim3(pass_grid(g, pk, smem));
  knp.blockDim = dim3(pk.threads);
  knp.sharedMemBytes = (unsigned)smem;
  knp.kernelParams = args;
  cudaGraphNode_t kn;
  e = cudaGraphAddKernelNode(&kn, body, nullptr, 0, &knp);
#if CUSHA_DIAG_COND_NODE
  if (e == cudaSuccess) {
    const Ctl* ctlp = g.d_ctl;
    void* cargs[] = {&ctlp, &handle};
    cudaKernelNodeParams cnp = {};
    cnp.func = reinterpret_cast<void*>(diag_set_cond);
    cnp.gridDim = dim3(1);
    cnp.blockDim = dim3(1);
    cnp.kernelParams = cargs;
    cudaGraphNode_t sn;
    e = cudaGraphAddKernelNode(&sn, body, &kn, 1, &cnp);
  }
#endif
  if (e == cudaSuccess) e = cudaGraphInstantiate(&h->exec[alg], graph, 0);
  cudaGraphDestroy(graph);
  if (e != cudaSuccess) { h->exec[alg] = nullptr; return fail(CUSHA_ECUDA, std::string("graph: ") + cudaGetErrorString(e)); }
  return CUSHA_OK;
}

int cusha_run(cusha_algorithm alg, cusha_graph* h, uint32_t source, uint32_t max_iters) {
  if (!h) return fail(CUSHA_EINVAL, "graph is NULL");
  if ((int)alg < 0 || (int)alg >= kNumAlgs) return fail(CUSHA_EINVAL, "bad algorithm");
  Graph& g = h->g;
  const int a = (int)alg;
  if ((a == kBFS || a == kSSSP || a == kSSWP) && source >= g.V) return fail(CUSHA_EINVAL, "source >= num_vertices");
  if (alg_needs_edge_values(a) && !g.has_ev) return fail(CUSHA_EINVAL, "algorithm needs edge_values");
  if (alg_needs_init(a) && !g.d_init[a]) return fail(CUSHA_EINVAL, "NN/HS/CS need cusha_set_vertex_values first");
  CKA(cudaSetDevice(g.device));
  // trace buffer sized to min(max_iters, 2^20)
  const uint32_t want_cap = std::min<uint32_t>(std::max<uint32_t>(max_iters, 1), 1u << 20);
  if (g.trace_cap < want_cap) {
    if (g.d_trace) cudaFreeAsync(g.d_trace, g.stream);
    g.d_trace = nullptr;
    g.trace_cap = 0;
    CKA(cudaMallocAsync(&g.d_trace, sizeof(TraceRec) * (size_t)want_cap, g.stream));
    CKA(cudaMemsetAsync(g.d_trace, 0, sizeof(TraceRec) * (size_t)want_cap, g.stream));
    g.trace_cap = want_cap;
    g.trace_dirty = 0;
    for (auto& e : h->exec)  // kernel params captured the old trace pointer
      if (e) { cudaGraphExecDestroy(e); e = nullptr; }
  }
  const PassKernel& pk = pass_kernel(a, g.repr);
  size_t smem = 0;
  int mapj = 0, stash = 0;
  uint32_t nst = 0;
  int rc = pass_config(g, pk, &smem, &mapj, &stash, &nst);
  if (rc) return rc;
  const bool host_loop = g.host_loop || g.G > 1;  // the partitioned mode exchanges between passes
  // overlapped passes (default): one launch runs every pass; it needs a trace
  // record per pass (<= 2^20), else the CUDA-graph loop runs one launch per pass
  // automatic mode: many small shards per CTA favour one launch per pass
  // (67_16 at |N| = 1536: 4.40 vs 5.48 ms)
  bool barrier = g.pass_barrier == 1;
  if (g.pass_barrier == 0 && g.S) {
    const uint64_t grid = pass_grid(g, pk, smem);
    barrier = (uint64_t)g.S >= 16 * grid && g.P <= 16384ull * g.S;
  }
  const bool multi = !host_loop && !barrier && max_iters <= g.trace_cap;
  if (!host_loop && !multi) {
    rc = ensure_exec(h, a);
    if (rc) return rc;
  }
  // records a previous run may have written (the rest are still zero)
  if (g.trace_dirty) CKA(cudaMemsetAsync(g.d_trace, 0, sizeof(TraceRec) * (size_t)g.trace_dirty, g.stream));
  g.trace_dirty = g.trace_cap;  // until this run's extent is known
  CKA(cudaEventRecord(g.ev0, g.stream));
  CKA(launch_reset_ctl(g.d_ctl, max_iters, g.stream));
  CKA(launch_init(g, a, source, g.stream));
  CKA(cudaEventRecord(g.evm, g.stream));
  if (max_iters > 0 && multi) {
    KParams kp = make_params(g, source);
    kp.multi = 1;
    kp.mapj = mapj;
    kp.stash = stash;
    kp.nst = nst;
    kp.ahead = pass_ahead(g, a);
    void* args[] = {&kp};
    CKA(cudaLaunchKernel(pk.func, dim3(pass_grid(g, pk, smem)), dim3(pk.threads), args, smem, g.stream));
  } else if (max_iters > 0 && !host_loop) {
    CKA(cudaGraphLaunch(h->exec[a], g.stream));
  }
  if (max_iters > 0 && host_loop) {
    // passes launched by the host in chunks; a pass that finds the run
    // converged (or at max_iters) exits at once, so over-launching is exact.
    // Partitioned: pass -> exchange (NCCL, multi-GPU) -> refresh of remote
    // windows + global convergence; every rank takes the same decisions
    // from the same exchanged data, so all issue the same collectives.
    KParams kp = make_params(g, source);
    kp.mapj = mapj;
    kp.stash = stash;
    kp.nst = nst;
    kp.ahead = pass_ahead(g, a);
    void* args[] = {&kp};
    const dim3 grid(pass_grid(g, pk, smem));
    // 8 passes per host check, multi-GPU too: a pass launched after the run
    // converged exits at once and the exchange / refresh after it change
    // nothing, and every rank reads the same convergence flag after the same
    // chunk, so all ranks issue the same collectives
    const int chunk = 8;
    std::string err;
    for (;;) {
      for (int k = 0; k < chunk; ++k) {
        CKA(cudaLaunchKernel(pk.func, grid, dim3(pk.threads), args, smem, g.stream));
        if (g.G > 1) {
          if (!g.simulate && (rc = nccl_exchange(g, 0, false, err))) return fail(rc, "exchange: " + err);
          CKA(launch_refresh(g, g.stream));
        }
      }
      CKA(cudaMemcpyAsync(g.h_ctl, g.d_ctl, sizeof(Ctl), cudaMemcpyDeviceToHost, g.stream));
      CKA(cudaStreamSynchronize(g.stream));
      if (g.h_ctl->converged || g.h_ctl->iter >= max_iters) break;
    }
    if (g.G > 1 && !g.simulate && (rc = nccl_exchange(g, (uint32_t)value_bytes(a), true, err)))
      return fail(rc, "final exchange: " + err);
  }
  CKA(cudaEventRecord(g.ev1, g.stream));
  CKA(cudaMemcpyAsync(g.h_ctl, g.d_ctl, sizeof(Ctl), cudaMemcpyDeviceToHost, g.stream));
  CKA(cudaStreamSynchronize(g.stream));
  float ms = 0, lms = 0;
  cudaEventElapsedTime(&ms, g.ev0, g.ev1);
  cudaEventElapsedTime(&lms, g.evm, g.ev1);
  Ctl c = *g.h_ctl;
  {  // passes whose trace records this run touched: its iterations, or every drawn ticket's pass
    const uint64_t drawn = multi && g.S ? c.ticket / g.S + 1 : 0;
    g.trace_dirty = (uint32_t)std::min<uint64_t>(g.trace_cap, std::max<uint64_t>(c.iter, drawn) + 2);
  }
  if (multi && max_iters > 0) {  // the confirming pass that committed nothing, else max_iters passes ran
    c.converged = c.conv_iter != 0xFFFFFFFFu;
    c.iter = c.converged ? c.conv_iter : max_iters;
  }
  // statistics and algorithmic bytes
  const uint64_t vb = value_bytes(a);
  const uint64_t evb = alg_needs_edge_values(a) ? 4 : 0;
  const uint32_t n = std::min(c.iter, g.trace_cap);
  TraceRec* tr = new TraceRec[n ? n : 1];
  CKA(cudaMemcpy(tr, g.d_trace, sizeof(TraceRec) * n, cudaMemcpyDeviceToHost));
  uint64_t bytes = 0, edges = 0;
  for (uint32_t i = 0; i < n; ++i) {
    // vertices of the processed shards (all of V unless clean shards were skipped)
    const uint64_t nv = std::min<uint64_t>(g.V, tr[i].shards * (uint64_t)g.N);
    bytes += nv * vb + (a == kPR ? 4ull * nv : 0);                    // stages 1+3 reads
    bytes += (uint64_t)tr[i].updated * vb;                            // stage 3 commits
    bytes += tr[i].edges * (4 + 2 + evb);                             // stage 2
    edges += tr[i].edges;
    if (g.repr == CUSHA_REPR_CW)  // SrcIndexCW + window index (+ delta row) or u32 Mapper; SrcValue
      bytes += tr[i].wb_entries * (mapj ? 4 : 6) + tr[i].wb_stores * 4 +
               (mapj ? (uint64_t)tr[i].shards * 4ull * g.S : 0);
    else
      bytes += tr[i].wb_entries * 4 + tr[i].wb_stores * 4 + (uint64_t)tr[i].active_shards * 8ull * g.S;
  }
  delete[] tr;
  g.st.iterations = c.iter;
  g.st.converged = c.converged;
  g.st.run_ms = ms;
  g.st.loop_ms = lms;
  g.st.last_algorithm = a;
  g.st.algorithmic_bytes = bytes;
  g.st.edges_processed = n == c.iter ? edges : (uint64_t)c.iter * g.E;
  g.st.stage2_bytes_per_iter = g.E * (4 + 2 + evb);
  g.st.wb_bytes_all_active = g.repr == CUSHA_REPR_CW ? g.E * (mapj ? 8 : 10) : g.E * 8;
  g.st.mapper_form = (uint32_t)mapj;
  g.st.device_loop = host_loop ? 0 : (multi ? 2 : 1);
  g.last_alg = a;
  g.have_values = true;
  return c.converged ? CUSHA_OK : CUSHA_NOT_CONVERGED;
}

int cusha_get_values(const cusha_graph* h, void* out, size_t out_bytes) {
  if (!h || !out) return fail(CUSHA_EINVAL, "null argument");
  const Graph& g = h->g;
  if (!g.have_values) return fail(CUSHA_ESTATE, "no run yet");
  const size_t want = (size_t)g.V * value_bytes(g.last_alg);
  if (out_bytes != want) return fail(CUSHA_EINVAL, "out_bytes must be |V| * value_bytes(last algorithm)");
  CKA(cudaSetDevice(g.device));
  CKA(cudaMemcpyAsync(out, g.d_vv, want, cudaMemcpyDeviceToHost, g.stream));
  CKA(cudaStreamSynchronize(g.stream));
  return CUSHA_OK;
}

int cusha_get_values_device(const cusha_graph* h, void* dptr, size_t out_bytes) {
  if (!h || !dptr) return fail(CUSHA_EINVAL, "null argument");
  const Graph& g = h->g;
  if (!g.have_values) return fail(CUSHA_ESTATE, "no run yet");
  const size_t want = (size_t)g.V * value_bytes(g.last_alg);
  if (out_bytes != want) return fail(CUSHA_EINVAL, "out_bytes must be |V| * value_bytes(last algorithm)");
  CKA(cudaSetDevice(g.device));
  CKA(cudaMemcpyAsync(dptr, g.d_vv, want, cudaMemcpyDeviceToDevice, g.stream));
  CKA(cudaStreamSynchronize(g.stream));
  return CUSHA_OK;
}

int cusha_get_stats(const cusha_graph* h, cusha_stats* s) {
  if (!h || !s) return fail(CUSHA_EINVAL, "null argument");
  *s = h->g.st;
  return CUSHA_OK;
}

int cusha_get_trace(const cusha_graph* h, uint32_t* upd, uint32_t* act, uint32_t cap) {
  if (!h) return fail(CUSHA_EINVAL, "null argument");
  const Graph& g = h->g;
  if (!g.have_values || !g.d_trace) return 0;
  const uint32_t n = std::min(std::min(g.st.iterations, g.trace_cap), cap);
  if (!n) return 0;
  TraceRec* tr = new TraceRec[n];
  cudaSetDevice(g.device);
  if (cudaMemcpy(tr, g.d_trace, sizeof(TraceRec) * n, cudaMemcpyDeviceToHost) != cudaSuccess) {
    delete[] tr;
    return fail(CUSHA_ECUDA, "trace copy");
  }
  for (uint32_t i = 0; i < n; ++i) {
    if (upd) upd[i] = tr[i].updated;
    if (act) act[i] = tr[i].active_shards;
  }
  delete[] tr;
  return (int)n;
}

int cusha_get_layout(const cusha_graph* h, cusha_layout_part part, void* out, size_t out_bytes, uint64_t* count) {
  if (!h) return fail(CUSHA_EINVAL, "graph is NULL");
  const Graph& g = h->g;
  const void* src = nullptr;
  const void* tail = nullptr;  // host-resident part (row f3) from position `split`
  uint64_t n = 0, split = ~0ull;
  size_t es = 4;
  switch (part) {
    case CUSHA_LAYOUT_SHARD_OFFSETS: src = g.d_shard_off; n = (uint64_t)g.S + 1; break;
    case CUSHA_LAYOUT_SHARD_SIZES: src = g.d_shard_cnt; n = g.S; break;
    case CUSHA_LAYOUT_SRC_INDEX: src = g.d_srcloc; tail = g.h_srcloc; split = g.splitP; n = g.P; es = 2; break;
    case CUSHA_LAYOUT_DEST_LOCAL: src = g.d_dest; tail = g.h_dest; split = g.splitP; n = g.P; es = 2; break;
    case CUSHA_LAYOUT_EDGE_ID: src = g.d_eid; tail = g.h_eid; split = g.splitP; n = g.P; break;
    case CUSHA_LAYOUT_WINDOWS: src = g.d_win; n = ((uint64_t)g.S + 1) * g.S; break;
    case CUSHA_LAYOUT_CW_OFFSETS: src = g.d_cw_off; n = (uint64_t)g.S + 1; break;
    case CUSHA_LAYOUT_CW_SIZES: src = g.d_cw_cnt; n = g.S; break;
    case CUSHA_LAYOUT_CW_SRC_LOCAL: src = g.d_cw_src; tail = g.h_cw_src; split = g.splitQ; n = g.Q; es = 2; break;
    case CUSHA_LAYOUT_MAPPER: src = g.d_mapper; tail = g.h_mapper; split = g.splitQ; n = g.Q; break;
    case CUSHA_LAYOUT_OUT_DEGREE: src = g.d_outdeg; n = g.V; break;
    case CUSHA_LAYOUT_RUN_K: src = g.d_run_k; n = g.R; break;
    case CUSHA_LAYOUT_RUN_T: src = g.d_run_t; n = g.R; break;
    case CUSHA_LAYOUT_CW_WINDOW: src = g.d_cw_win; tail = g.h_cw_win; split = g.splitQ; n = g.Q; es = 2; break;
    case CUSHA_LAYOUT_CW_DELTA: src = g.d_cw_delta; n = (uint64_t)g.S * g.S; break;
    default: return fail(CUSHA_EINVAL, "bad layout part");
  }
  if (!src && !tail) return fail(CUSHA_EUNSUPPORTED, "part not held by this representation");
  if (count) *count = n;
  if (!out) return CUSHA_OK;
  if (out_bytes < n * es) return fail(CUSHA_EINVAL, "out_bytes too small");
  CKA(cudaSetDevice(g.device));
  const uint64_t nd = std::min(n, split);  // HBM part
  if (nd) CKA(cudaMemcpy(out, src, nd * es, cudaMemcpyDeviceToHost));
  if (nd < n) std::memcpy(static_cast<char*>(out) + nd * es, tail, (n - nd) * es);
  return CUSHA_OK;
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
  const Graph& g = h->g;
  if (g.G <= 1) {
    if (cap < 2) return fail(CUSHA_EINVAL, "cap too small");
    bounds[0] = 0;
    bounds[1] = g.S;
    return 1;
  }
  if (cap < g.G + 1) return fail(CUSHA_EINVAL, "cap too small");
  for (uint32_t q = 0; q <= g.G; ++q) bounds[q] = g.h_bounds[q];
  return (int)g.G;
}

int cusha_diag_timeline(void* out, size_t out_bytes) {
  if (!out) return fail(CUSHA_EINVAL, "null argument");
  cudaDeviceSynchronize();
  const int n = timeline_copy(out, out_bytes);
  return n < 0 ? fail(CUSHA_EUNSUPPORTED, "library built without CUSHA_TIMELINE") : n;
}

}  // extern "C"
