// graph.hpp — internal (non-ABI) declarations shared by the library's .cu files.
#pragma once
#include <cstddef>
#include <cstdint>
#include <string>
#include <vector>
#include <cuda_runtime.h>

#include "../../include/cusha.h"

namespace cusha {

constexpr uint32_t kRunUnit = 128;  // CW positions per entry of the Mapper-run locator (RunUnit)

// Iteration control word block (row a5), one per graph, device resident.
struct Ctl {
  uint32_t iter;        // shard passes completed in this run
  uint32_t changed;     // set by any CTA whose stage 3 committed an update (is_converged = false, L255)
  uint32_t ctas_done;   // arrival counter; the last CTA closes the iteration
  uint32_t max_iters;
  uint32_t converged;   // 1 once a pass committed nothing
  uint32_t next_shard;  // dynamic shard queue of the persistent pass
  uint32_t lchanged;    // partitioned mode: this partition's last pass committed an update
  uint32_t gchanged;    // partitioned mode: OR of lchanged over the partitions (NCCL all-reduce / simulation)
  // overlapped passes (one launch per run)
  unsigned long long ticket;  // shard tickets drawn: ticket t = shard t % |S| of pass t / |S|
  uint32_t stop;              // `window` consecutive passes committed nothing: draw no more tickets
  uint32_t conv_iter;         // 1 + the last of those passes (~0u: none yet)
};

// One process per GPU (row e): every rank's barrier block, in its own memory,
// mapped by the others (CUDA IPC).  Round r of the barrier uses slot r & 1.
struct PeerSync {
  uint32_t arrive[2];       // ranks that reached this round
  uint32_t round;           // barrier rounds this rank completed
  uint32_t err;             // 1: a peer did not arrive within the timeout
  uint32_t changed[2][64];  // rank q's "committed an update" word of this round
};

// Per-iteration trace (row f4; also the source of algorithmic byte counts).
struct TraceRec {
  uint32_t updated;          // vertices committed in stage 3
  uint32_t active_shards;    // shards that ran stage 4
  uint32_t done;             // overlapped passes: shard tickets of this pass completed
  uint32_t pad_;
  unsigned long long wb_entries;  // CW / window entries visited by stage 4
  unsigned long long wb_stores;   // SrcValue words actually stored by stage 4
  unsigned long long edges;       // edges streamed by stage 2 (|E| unless clean shards are skipped)
  unsigned long long shards;      // shards processed (|S| unless clean shards are skipped)
};

// Everything a shard-pass launch needs (passed by value).
// Arrays of one partition are indexed by the LOCAL shard index sl = s - s0
// (shard s is global; partition = shards [s0, s0 + Sl), vertices [s0*N,
// min(V, (s0+Sl)*N))); a single GPU is the partition s0 = 0, Sl = S.
struct KParams {
  uint32_t V, N, S, source;
  uint32_t s0, Sl;             // first shard and number of shards of this partition
  const uint32_t* shard_off;   // Sl+1 padded start positions (local positions)
  const uint32_t* shard_cnt;   // Sl real entry counts
  const uint16_t* dest;        // P local DestIndex (filler = N)
  const uint32_t* ev;          // P EdgeValue or null
  uint32_t* srcvalue;          // P+1 SrcValue of this partition's shard entries (read by stage 2)
  uint32_t* sv_write;          // single partition: where stage 4 writes (= srcvalue; the other buffer in BSP mode)
  uint32_t* const* sv_peer;    // G: SrcValue of every partition (sv_peer[own] = srcvalue); stage 4 of a
                               // source shard stores into the partition that owns each window's target
  const uint16_t* srcloc;      // GS: P SrcIndex - (source shard)*N
  const uint32_t* win;         // (Sl+1)*S window starts: rows s0..s0+Sl of the window table (GS walk, skip marks)
  const uint32_t* cw_off;      // CW: Sl+1 padded CW_i starts (own source shards i)
  const uint32_t* cw_cnt;      // Sl real |CW_i| (both reprs; = entries stage 4 of shard i visits)
  uint8_t* active;             // Sl: shard ran stage 4 in the last pass (stage-4 prefetch predictor)
  const uint16_t* cw_src;      // CW: Q local SrcIndex
  const uint32_t* mapper;      // CW: Q target positions in the owning partition's SrcValue
  const uint16_t* cw_win;      // CW: Q target shard j of each entry (filler: 0xFFFF)
  const uint32_t* cw_delta;    // CW: Sl*S, Mapper[k] = cw_delta[il*S + j] + k for k in W_ij's part of CW_i
  void* vv;                    // VertexValues of the partition's vertices (local index (s - s0)*N + v)
  const uint32_t* outdeg;      // out-degrees of the partition's vertices (PR NbrsNum)
  Ctl* ctl;
  TraceRec* trace;
  uint32_t trace_cap;
  int multi;                   // 1: one launch runs every pass (overlapped passes)
  uint32_t window;             // overlapped passes: pass k starts after pass k - window completed
  int mapj;                    // 1: CW stage 4 uses the Mapper in window form (cw_win + delta row in smem)
  int stash;                   // 1: integer algorithms keep stage 1's VertexValues in smem for stage 3
  int ahead;                   // 1: the producer prefetches stage-2 tiles into L2 beyond the ring (HBM-resident passes)
  uint32_t nst;                // ring slots of this run (kStages, or more when shared memory has room)
  uint32_t s4two;              // integer algorithms: two stage-4 entries per thread per step (one CTA per SM)
  uint32_t* shard_seq;         // Sl: passes of shard s completed (overlapped passes)
  const uint32_t* order;       // Sl: shard processed by the q-th ticket of a pass (nullptr: shard order)
  // destination-range partition (row e); G = 1: single partition
  uint32_t G;                  // partitions
  const uint32_t* bounds;      // G+1 shard bounds of the partitions
  const uint8_t* owner;        // S: partition owning shard j
  const uint32_t* cwp;         // Sl*(G+1): CW_i entries whose targets lie in partition q = [cwp[il][q], cwp[il][q+1])
  uint32_t* const* dirty_peer; // G: dirty[] of every partition (clean-shard skipping marks remote shards)
  // Mapper in run-length form (CW): one run per non-empty window
  const uint32_t* run_k;       // R (+pad): CW position of each run's first entry (sorted)
  const uint32_t* run_t;       // R (+pad): target shard position of that entry
  const uint32_t* run_unit;    // Q/kRunUnit+2: last run starting at or before u*kRunUnit
  const uint32_t* run_bits;    // Q/32 (+pad): bit k = a run starts at CW position k
  const uint32_t* run_d;       // R (+pad): RunT - RunK (mod 2^32): target(k) = k + run_d[run of k]
  uint32_t R;
  // opt-in exact work skipping
  int skip;                    // 1: a shard none of whose windows was written since its last pass is skipped
  uint32_t* dirty;             // Sl: some window of shard j written since j's last pass (set by writers)
  // host-streamed topology (row f3): entries at shard
  // positions >= splitP / CW positions >= splitQ live in pinned host memory
  // (x_h[i - split]); below the split, in HBM (x[i]).  splitP = P, splitQ = Q: all in HBM.
  uint32_t splitP, splitQ;
  const uint16_t* dest_h;
  const uint32_t* ev_h;
  const uint16_t* srcloc_h;
  const uint16_t* cw_src_h;
  const uint32_t* mapper_h;
  const uint16_t* cw_win_h;
};

// element i of a topology array split between HBM (i < split) and pinned host memory
template <class T>
__host__ __device__ __forceinline__ const T* topo_at(const T* dev, const T* host, uint32_t split, uint64_t i) {
  return i < split ? dev + i : host + (i - split);
}

struct PassKernel {
  const void* func;       // __global__ shard_pass<Alg, Repr>
  uint32_t words;         // shared 32-bit words per vertex (local state)
  bool wb_array;          // separate write-back value array in shared memory
  bool monotone;          // changed-bit array in shared memory
  uint32_t ring_bytes;    // TMA tile ring (the default kStages slots)
  uint32_t slot_bytes;    // one ring slot
  uint32_t max_stages;    // most slots a run may use
  uint32_t threads;       // CTA size (producer warp + consumer warps)
  bool persistent;        // grid = resident CTAs pulling shards from a queue (else one CTA per shard)
  size_t smem_bytes(uint32_t N, uint32_t delta_row = 0) const;  // delta_row: words of the window-form row
};

// One partition's device state (row a0 layout + per-run arrays).  A single
// GPU holds one partition covering every shard (s0 = 0, Sl = S); the
// destination-range partition of row e gives each rank (or, in the one-process
// simulation, each sub-graph) shards [s0, s0 + Sl) and their in-edges, plus the
// Concatenated Windows of its own SOURCE shards, whose Mapper targets are
// positions in the SrcValue array of the partition that owns each window.
struct Graph {
  // topology
  uint32_t V = 0, N = 0, S = 0;     // global |V|, |N|, |S|
  uint64_t E = 0, P = 0, Q = 0;     // E: global |E|; P, Q: this partition's padded shard / CW entries
  uint32_t s0 = 0, Sl = 0;          // owned shards [s0, s0 + Sl)
  uint32_t v0 = 0, nvl = 0;         // owned vertices [v0, v0 + nvl)
  uint64_t E_loc = 0;               // real in-edges of the owned shards
  int repr = 0, device = 0;
  cudaStream_t stream = nullptr;
  bool own_stream = false;
  bool has_ev = false;
  bool keep_ids = false;            // keep the input edge index per entry (layout inspection only)
  uint32_t* d_shard_off = nullptr;  // Sl+1
  uint32_t* d_shard_cnt = nullptr;  // Sl
  uint16_t* d_dest = nullptr;       // P
  uint16_t* d_srcloc = nullptr;     // P (GS): SrcIndex local to its source shard
  uint32_t* d_eid = nullptr;        // P (only with keep_ids)
  uint32_t* d_ev = nullptr;         // P (if has_ev)
  uint32_t* d_win = nullptr;        // (Sl+1)*S: rows s0..s0+Sl of the window table
  uint32_t* d_cw_off = nullptr;     // Sl+1
  uint32_t* d_cw_cnt = nullptr;     // Sl
  uint8_t* d_active = nullptr;      // Sl: stage-4 prefetch predictor
  uint32_t* d_dirty = nullptr;      // Sl: clean-shard skipping flags
  uint32_t* d_shard_seq = nullptr;  // Sl: overlapped passes, per-shard pass order
  uint32_t* d_order = nullptr;      // Sl: largest shards first (L2-resident passes; built on first use)
  uint2* d_init_chunks = nullptr;   // CW init: (shard, first CW position) per chunk of kInitChunk entries (first run)
  uint32_t init_nchunks = 0;
  int pass_barrier = 0;             // 0: automatic, 1: one launch per pass, 2: overlapped
  bool skip_clean = false;
  // host-streamed topology (row f3): shards >= host_shard keep their entry
  // arrays (and CW_i arrays) in pinned, mapped host memory
  uint64_t topo_budget = 0;         // HBM bytes allowed for per-entry topology; 0 = unlimited
  uint32_t host_shard = 0;          // first host-resident shard (S: none)
  uint64_t splitP = 0, splitQ = 0;  // shard / CW positions where host residency starts
  uint16_t* h_dest = nullptr;       // P - splitP   (pinned host, mapped)
  uint32_t* h_ev = nullptr;
  uint16_t* h_srcloc = nullptr;
  uint32_t* h_eid = nullptr;
  uint16_t* h_cw_src = nullptr;     // Q - splitQ
  uint32_t* h_mapper = nullptr;
  uint64_t host_bytes = 0;
  uint16_t* d_cw_src = nullptr;     // Q (CW)
  uint32_t* d_mapper = nullptr;     // Q (CW)
  uint16_t* d_cw_win = nullptr;     // Q (CW): target shard of each entry (Mapper in window form)
  uint32_t* d_cw_delta = nullptr;   // Sl*S (CW): Mapper - CW position, per window
  uint16_t* h_cw_win = nullptr;     // Q - splitQ (row f3)
  uint32_t R = 0;                   // Mapper runs (non-empty windows; CUSHA_RLE builds only)
  uint32_t* d_run_k = nullptr;      // R+pad
  uint32_t* d_run_t = nullptr;      // R+pad
  uint32_t* d_run_unit = nullptr;   // Q/kRunUnit+2
  uint32_t* d_run_bits = nullptr;   // Q/32 + pad
  uint32_t* d_run_d = nullptr;      // R+pad
  uint32_t* d_outdeg = nullptr;     // nvl
  uint32_t max_indeg = 0;           // largest in-degree (fixed-point range check)
  float max_abs_ev = 0.f;           // largest |EdgeValue| read as f32 (fixed-point range check)
  // per-run state
  uint32_t* d_srcvalue = nullptr;   // P+1
  bool srcvalue_ipc = false;        // allocated with cudaMalloc (exported to the other ranks)
  bool bsp = false;                 // two-phase BSP mode: stage 4 writes the next pass's SrcValue copy
  uint32_t* d_srcvalue2 = nullptr;  // BSP mode: the second SrcValue buffer
  void* d_vv = nullptr;             // nvl * 8 bytes
  void* d_init[8] = {};             // user initial values per algorithm (this partition's slice)
  float init_max_abs[8] = {};       // largest |initial value| given per algorithm
  Ctl* d_ctl = nullptr;
  TraceRec* d_trace = nullptr;
  uint32_t trace_cap = 0;
  uint32_t trace_dirty = 0;         // leading trace records a previous run may have written
  // host mirror (api.cu): the Ctl block, then the first kHostTrace trace
  // records, read back together at the end of a run
  Ctl* h_ctl = nullptr;
  TraceRec* h_trace = nullptr;
  void* h_mirror = nullptr;
  void (*mirror_deleter)(void*) = nullptr;
  void free_mirror() {
    if (h_mirror && mirror_deleter) mirror_deleter(h_mirror);
    h_mirror = nullptr;
    h_ctl = nullptr;
    h_trace = nullptr;
  }
  cudaEvent_t ev0 = nullptr, ev1 = nullptr, evm = nullptr;  // run timing (created once per graph)
  // destination-range partition (row e)
  int world_size = 1, rank = 0;
  uint32_t G = 1;                   // partitions (1: unpartitioned)
  uint32_t part = 0;                // this partition's index
  std::vector<uint32_t> h_bounds;   // G+1 shard bounds
  uint32_t* d_bounds = nullptr;     // G+1
  uint8_t* d_owner = nullptr;       // S
  uint32_t* d_cwp = nullptr;        // Sl*(G+1)
  uint32_t** d_sv_peer = nullptr;   // G: SrcValue of every partition (device pointers valid on this device)
  uint32_t** d_dirty_peer = nullptr;// G: dirty[] of every partition (skip_clean only)
  PeerSync* d_sync = nullptr;       // one process per GPU: this rank's barrier block (cudaMalloc, exported)
  PeerSync** d_sync_peer = nullptr; // G: every rank's barrier block
  std::vector<void*> vv_peer;       // G: every rank's VertexValues (for cusha_get_values)
  bool connected = false;           // peers mapped (multi-process modes)
  std::vector<void*> ipc_open;      // peer allocations mapped with cudaIpcOpenMemHandle
  void* nccl_comm = nullptr;        // ncclComm_t (real multi-GPU)
  uint32_t comm_timeout_ms = 300000;
  // stats
  cusha_stats st{};
  int last_alg = -1;
  bool have_values = false;
  bool host_loop = false;
};

// kernels.cu
const PassKernel& pass_kernel(int alg, int repr);
// CW entries per block of the SrcValue initialisation (one partition, G = 1)
constexpr uint32_t kInitChunk = 1024;
cudaError_t launch_init(const Graph& g, int alg, uint32_t source, cudaStream_t s);
cudaError_t launch_reset_ctl(Ctl* ctl, uint32_t max_iters, cudaStream_t s);
cudaError_t launch_close_parts(Ctl* const* ctls, uint32_t G, cudaStream_t s);  // partitioned: global convergence
// one process per GPU: barrier over the ranks' PeerSync blocks; decide = also
// OR the ranks' lchanged words into the convergence flag
cudaError_t launch_peer_barrier(const Graph& g, int decide, uint32_t timeout_ms, cudaStream_t s);
KParams make_params(const Graph& g, uint32_t source);
size_t value_bytes(int alg);
int timeline_copy(void* out, size_t bytes);  // CUSHA_TIMELINE builds: per-ticket stamps (else -1)
bool kernels_rle();  // built with the Mapper-runs stage 4 (CUSHA_RLE)

bool alg_needs_edge_values(int alg);
bool alg_needs_init(int alg);

// builder.cu
// Host inputs copied in chunks on a copy stream (row f2): chunk c = edges
// [bounds[c], bounds[c+1]) of src/dst is on the device once ready[c] fired;
// `all` fires after every copy (edge values included).
struct InputChunks {
  int n = 0;
  uint64_t bounds[17] = {};
  cudaEvent_t ready[16] = {};
  cudaEvent_t all = nullptr;
};
int build_layout(Graph& g, const uint32_t* d_src, const uint32_t* d_dst, const uint32_t* d_val, std::string& err,
                 const InputChunks* chunks = nullptr);
int build_runs(Graph& g, std::string& err);       // Mapper runs (CW, CUSHA_RLE builds)
int offload_topology(Graph& g, std::string& err); // row f3: move shards >= host_shard to pinned host memory
void partition_bounds(uint32_t S, const uint64_t* work, uint32_t G, uint32_t* bounds);
void free_device_arrays(Graph& g);  // every device / pinned array of g (not its stream or events)

// partition.cu: the per-partition layout built straight from the edge list
struct PlanInput {
  uint32_t V = 0, N = 0;
  uint64_t E = 0;
  const uint32_t *src = nullptr, *dst = nullptr, *val = nullptr;  // host or device
  bool host = false;
  cudaStream_t stream = nullptr;
};
struct Plan {  // from the shard-pair counts C[i][j] = |W_ij|
  uint32_t V = 0, N = 0, S = 0;
  uint64_t E = 0;
  uint32_t* d_C = nullptr;        // S*S
  uint32_t* d_win = nullptr;      // (S+1)*S: start of W_ij in shard j, local to j's partition
  uint32_t* d_R = nullptr;        // S*S: start of W_ij inside CW_i
  uint32_t* d_outdeg = nullptr;   // V
  std::vector<uint32_t> in, out;  // entries per shard (its in-edges) / per CW_i (its vertices' out-edges)
  std::vector<uint32_t> bounds;   // G+1
  std::vector<uint8_t> owner;     // S
  std::vector<uint32_t> offl, coffl;  // padded offset of shard j / CW_i inside its partition
  uint32_t max_indeg = 0;
  float max_abs_ev = 0.f;
};
int plan_partitions(const PlanInput& in, uint32_t G, Plan& plan, std::string& err);
void free_plan(Plan& plan, cudaStream_t st);
int build_part_direct(const PlanInput& in, const Plan& plan, uint32_t r, Graph& part, std::string& err);
cudaError_t dev_alloc(void** p, size_t bytes, cudaStream_t s);  // the library's private stream-ordered pool
cudaError_t trim_pool(int dev);                                  // release its unused blocks

// api.cu
void set_error(const std::string& msg);

// nccl.cu (loaded at run time; no link-time NCCL dependency)
int nccl_unique_id(void* out128, std::string& err);
int nccl_init(Graph& g, const void* id128, std::string& err);
int nccl_allgather_bytes(Graph& g, const void* dsend, void* drecv, size_t bytes, std::string& err);
int nccl_wait(Graph& g, uint32_t timeout_ms, std::string& err);  // stream drained, or abort on error / timeout
void nccl_destroy(Graph& g);

}  // namespace cusha
