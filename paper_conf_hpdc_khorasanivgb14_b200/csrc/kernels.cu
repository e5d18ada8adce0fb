// kernels.cu — the shard pass (rows a1-a5) and its initialisation kernels.
//
// One launch = one CuSha iteration (Fig. 5): one CTA per shard
// (L191), four stages separated by block barriers, and the global
// convergence flag (L189, L255).  The iteration loop itself stays on the
// device: the last CTA to finish closes the iteration and sets the CUDA-graph
// while-condition, instead of the paper's
// per-iteration cudaMemcpy of is_converged (L189).
//
// B200 structure of a CTA: one producer warp drives the TMA engine
// (cp.async.bulk) to stream the shard's entry arrays — and, in stage 4, the
// CW_s index arrays — through a ring of kStages shared-memory tiles guarded
// by mbarriers; eight consumer warps reduce from / scatter out of the ring.
// The memory system thus sees kStages tiles in flight per CTA regardless of
// how long the consumers' shared-memory atomics take.
#include <cstdio>

#include "algorithms.cuh"
#include "graph.hpp"

namespace cusha {

constexpr uint32_t kFull = 0xFFFFFFFFu;
constexpr uint32_t kConsumerWarps = 8;
constexpr uint32_t kConsumers = kConsumerWarps * 32;
constexpr uint32_t kPassThreads = kConsumers + 32;  // + 1 producer warp
constexpr uint32_t kTile = 1024;                    // entries per ring slot
constexpr uint32_t kStages = 4;                     // ring depth

// ring slot: stage 2 = SrcValue (4T) | DestIndex (2T) | EdgeValue (4T);
//            stage 4 = SrcIndexCW (2T) | Mapper (4T)
template <class A>
constexpr uint32_t slot_bytes() {
  return kTile * (6 + (A::kEdge ? 4 : 0));
}

// ------------------------------------------------------------ stage 2 body
template <class A>
__device__ __forceinline__ void proc4(uint32_t* sm, uint32_t st, const uint4& sv, const uint2& dd, const uint4& ev) {
  const uint32_t D[4] = {dd.x & 0xFFFFu, dd.x >> 16, dd.y & 0xFFFFu, dd.y >> 16};
  const uint32_t S[4] = {sv.x, sv.y, sv.z, sv.w};
  const uint32_t W[4] = {ev.x, ev.y, ev.z, ev.w};
  if constexpr (A::kAcc == 0) {
#pragma unroll
    for (int k = 0; k < 4; ++k) A::compute(sm, st, D[k], S[k], W[k]);  // non-returning ATOMS.MIN/MAX
  } else {
    uint64_t F[4][2];
#pragma unroll
    for (int k = 0; k < 4; ++k) A::contrib(sm, st, D[k], S[k], W[k], F[k]);
    uint32_t old[4][2];
#pragma unroll
    for (int k = 0; k < 4; ++k)
#pragma unroll
      for (int a = 0; a < A::kAcc; ++a) old[k][a] = atomicAdd(&sm[A::acc_lo(a) * st + D[k]], (uint32_t)F[k][a]);
#pragma unroll
    for (int k = 0; k < 4; ++k)
#pragma unroll
      for (int a = 0; a < A::kAcc; ++a) {
        const uint32_t l = (uint32_t)F[k][a];
        const uint32_t h = (uint32_t)(F[k][a] >> 32) + ((old[k][a] + l < old[k][a]) ? 1u : 0u);  // carry
        if (h) atomicAdd(&sm[(A::acc_lo(a) + 1) * st + D[k]], h);
      }
  }
}

// stage-4 value of local vertex l and whether it must be stored
template <class A>
__device__ __forceinline__ bool wb_get(const uint32_t* sm, const uint32_t* aux, uint32_t l, uint32_t& val) {
  if (A::kMonotone) {
    // integer algorithms: local == committed value whenever not updated, so
    // copies of unchanged vertices already hold it (R19) — store only changed
    val = sm[l];
    return (aux[l >> 5] >> (l & 31)) & 1u;
  } else {
    val = aux[l];  // local_vertices as left by update_condition (Fig. 5 line 25)
    return true;
  }
}

// ------------------------------------------------- G-Shards window walker
// Visits every entry of the windows W_sj (j = 0..S-1) of source shard s:
// each warp takes 32 windows at a time, scans their lengths across lanes and
// walks the concatenation with one entry per lane (4 in flight), finding each
// entry's window by a 5-step binary search over the lanes' prefix sums.
// fn(e, l): e = shard position, l = SrcIndex - s*N.
template <class Fn>
__device__ __forceinline__ void gs_walk(const KParams& p, uint32_t s, uint32_t lane, uint32_t warp, uint32_t nwarps,
                                        Fn&& fn) {
  const uint32_t* r0 = p.win + (size_t)s * p.S;
  const uint32_t* r1 = r0 + p.S;
  for (uint32_t jb = warp * 32; jb < p.S; jb += nwarps * 32) {
    const uint32_t j = jb + lane;
    uint32_t a = 0, b = 0;
    if (j < p.S) { a = __ldg(r0 + j); b = __ldg(r1 + j); }
    const uint32_t len = b - a;
    uint32_t inc = len;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t t = __shfl_up_sync(kFull, inc, o);
      if (lane >= (uint32_t)o) inc += t;
    }
    const uint32_t total = __shfl_sync(kFull, inc, 31);
    const uint32_t exc = inc - len;
    for (uint32_t f0 = 0; f0 < total; f0 += 128) {
      uint32_t e[4], l[4];
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        const uint32_t f = f0 + u * 32 + lane;
        int w = 0;
#pragma unroll
        for (int step = 16; step; step >>= 1) {
          const uint32_t ex = __shfl_sync(kFull, exc, w + step);
          if (ex <= f) w += step;
        }
        e[u] = __shfl_sync(kFull, a, w) + (f - __shfl_sync(kFull, exc, w));
        l[u] = f < total ? (uint32_t)__ldg(p.srcloc + e[u]) : 0xFFFFFFFFu;
      }
#pragma unroll
      for (int u = 0; u < 4; ++u)
        if (l[u] != 0xFFFFFFFFu) fn(e[u], l[u]);
    }
  }
}

template <class A, int REPR>
__global__ void __launch_bounds__(kPassThreads, 2) shard_pass(const KParams p) {
  extern __shared__ __align__(128) uint8_t dyn[];
  constexpr uint32_t SLOT = slot_bytes<A>();
  uint8_t* const ring = dyn;
  uint32_t* const sm = reinterpret_cast<uint32_t*>(dyn + kStages * SLOT);
  __shared__ uint64_t full_bar[kStages], empty_bar[kStages];
  __shared__ uint32_t s_upd;
  __shared__ unsigned long long s_stores;
  using V_t = typename A::Value;
  const uint32_t tid = threadIdx.x, lane = tid & 31u, warp = tid >> 5;
  const uint32_t s = blockIdx.x, N = p.N, st = N + 1;
  const uint32_t off = s * N;
  const uint32_t nv = min(N, p.V - off);
  V_t* vv = reinterpret_cast<V_t*>(p.vv) + off;
  uint32_t* aux = sm + A::kWords * st;  // write-back values (float algs) or changed bits (integer algs)
  const uint32_t it = *reinterpret_cast<volatile uint32_t*>(&p.ctl->iter);
  // a pass launched after the run converged / hit max_iters is a no-op (host-loop mode)
  if (*reinterpret_cast<volatile uint32_t*>(&p.ctl->converged) || it >= p.ctl->max_iters) return;
  if (tid == 0) {
    s_upd = 0;
    s_stores = 0;
    for (uint32_t i = 0; i < kStages; ++i) {
      mbar_init(&full_bar[i], 1);                // the producer's arrive.expect_tx
      mbar_init(&empty_bar[i], kConsumerWarps);  // one arrive per consumer warp
    }
    mbar_fence_init();
  }

  // ---- stage 1: local_vertices <- init_compute(VertexValues) (Fig. 5 lines 8-10, L267)
  for (uint32_t v = tid; v < nv; v += kPassThreads) A::init(sm, st, v, vv[v]);
  if (tid == 0) A::init(sm, st, N, V_t{});  // trash slot for filler entries
  __syncthreads();

  // ring position: the producer lane and every consumer thread walk the same tile sequence
  uint32_t slot = 0, ph = 0;
  const uint32_t ct = tid - 32;  // consumer thread index (warps 1..8)

  // ---- stage 2: stream the shard's entries, compute() into shared memory (lines 12-13, L269)
  {
    const uint32_t b = p.shard_off[s], e = p.shard_off[s + 1];
    if (warp == 0) {
      if (lane == 0) {
        for (uint32_t t0 = b; t0 < e; t0 += kTile) {
          const uint32_t n = min(kTile, e - t0);
          mbar_wait(&empty_bar[slot], ph ^ 1);
          uint8_t* buf = ring + slot * SLOT;
          mbar_expect_tx(&full_bar[slot], n * (A::kEdge ? 10u : 6u));
          bulk_g2s(buf, p.srcvalue + t0, n * 4, &full_bar[slot]);
          bulk_g2s(buf + 4 * kTile, p.dest + t0, n * 2, &full_bar[slot]);
          if (A::kEdge) bulk_g2s(buf + 6 * kTile, p.ev + t0, n * 4, &full_bar[slot]);
          if (++slot == kStages) { slot = 0; ph ^= 1; }
        }
      }
    } else {
      for (uint32_t t0 = b; t0 < e; t0 += kTile) {
        const uint32_t n = min(kTile, e - t0);
        mbar_wait(&full_bar[slot], ph);
        const uint8_t* buf = ring + slot * SLOT;
        for (uint32_t i = ct * 4; i < n; i += kConsumers * 4) {
          const uint4 sv = *reinterpret_cast<const uint4*>(buf + 4 * i);
          const uint2 dd = *reinterpret_cast<const uint2*>(buf + 4 * kTile + 2 * i);
          uint4 ev = make_uint4(0, 0, 0, 0);
          if (A::kEdge) ev = *reinterpret_cast<const uint4*>(buf + 6 * kTile + 4 * i);
          proc4<A>(sm, st, sv, dd, ev);
        }
        __syncwarp();
        if (lane == 0) mbar_arrive(&empty_bar[slot]);
        if (++slot == kStages) { slot = 0; ph ^= 1; }
      }
    }
  }
  __syncthreads();

  // ---- stage 3: update_condition, commit to VertexValues, values_updated (lines 15-20, L271)
  uint32_t my_upd = 0;
  for (uint32_t base = 0; base < nv; base += kPassThreads) {
    const uint32_t v = base + tid;
    bool u = false;
    if (v < nv) {
      V_t out;
      uint32_t wbv = 0;
      const uint32_t od = A::kOutDeg ? __ldg(p.outdeg + off + v) : 0u;
      u = A::update(sm, st, v, vv[v], &out, &wbv, od);
      if (u) vv[v] = out;
      if (!A::kMonotone) aux[v] = wbv;
    }
    const uint32_t m = __ballot_sync(kFull, u);
    if (lane == 0 && m) atomicAdd(&s_upd, (uint32_t)__popc(m));
    if (A::kMonotone && lane == 0 && base + warp * 32 < nv) aux[(base >> 5) + warp] = m;
    my_upd |= u ? 1u : 0u;
  }
  const int any = __syncthreads_or((int)my_upd);

  // ---- stage 4: write-back into every shard's window (lines 23-26, L308)
  if (any) {
    uint32_t stores = 0;
    if (REPR == CUSHA_REPR_CW) {
      // thread per CW_s entry: SrcValue[Mapper[k]] = local[SrcIndex[k]] (L177,
      // Fig. 4b).  CW_s's index arrays stream through the ring; consecutive
      // consumer threads take consecutive entries, so the stores of one window
      // (consecutive Mapper targets) coalesce into whole sectors.
      const uint32_t kb = p.cw_off[s], ke = p.cw_off[s + 1];
      const uint32_t trash = p.shard_off[p.S];
      if (warp == 0) {
        if (lane == 0) {
          for (uint32_t k0 = kb; k0 < ke; k0 += kTile) {
            const uint32_t n = min(kTile, ke - k0);
            mbar_wait(&empty_bar[slot], ph ^ 1);
            uint8_t* buf = ring + slot * SLOT;
            mbar_expect_tx(&full_bar[slot], n * 6u);
            bulk_g2s(buf, p.cw_src + k0, n * 2, &full_bar[slot]);
            bulk_g2s(buf + 2 * kTile, p.mapper + k0, n * 4, &full_bar[slot]);
            if (++slot == kStages) { slot = 0; ph ^= 1; }
          }
        }
      } else {
        for (uint32_t k0 = kb; k0 < ke; k0 += kTile) {
          const uint32_t n = min(kTile, ke - k0);
          mbar_wait(&full_bar[slot], ph);
          const uint16_t* L = reinterpret_cast<const uint16_t*>(ring + slot * SLOT);
          const uint32_t* M = reinterpret_cast<const uint32_t*>(ring + slot * SLOT + 2 * kTile);
          for (uint32_t i = ct; i < n; i += kConsumers) {
            const uint32_t m = M[i];
            uint32_t val;
            if (m != trash && wb_get<A>(sm, aux, L[i], val)) { st_u32(p.srcvalue + m, val); ++stores; }
          }
          __syncwarp();
          if (lane == 0) mbar_arrive(&empty_bar[slot]);
          if (++slot == kStages) { slot = 0; ph ^= 1; }
        }
      }
    } else if (warp > 0) {
      // G-Shards: windows W_sj of every shard j (L151, Fig. 3c), walked a
      // batch of 32 windows per warp with one entry per lane (gs_walk)
      gs_walk(p, s, lane, warp - 1, kConsumerWarps, [&](uint32_t e, uint32_t l) {
        uint32_t val;
        if (wb_get<A>(sm, aux, l, val)) { st_u32(p.srcvalue + e, val); ++stores; }
      });
    }
#pragma unroll
    for (int o = 16; o; o >>= 1) stores += __shfl_xor_sync(kFull, stores, o);
    if (lane == 0 && stores) atomicAdd(&s_stores, (unsigned long long)stores);
    __syncthreads();
  }

  // ---- convergence flag and iteration close (line 26 "is_converged = false"; L189)
  if (tid == 0) {
    if (any) {
      *reinterpret_cast<volatile uint32_t*>(&p.ctl->changed) = 1u;
      if (it < p.trace_cap) {
        TraceRec* t = p.trace + it;
        atomicAdd(&t->updated, s_upd);
        atomicAdd(&t->active_shards, 1u);
        atomicAdd(&t->wb_entries, (unsigned long long)p.cw_cnt[s]);
        atomicAdd(&t->wb_stores, s_stores);
      }
    }
    __threadfence();
    const uint32_t t = atomicAdd(&p.ctl->ctas_done, 1u);
    if (t == gridDim.x - 1) {
      __threadfence();
      const uint32_t changed = *reinterpret_cast<volatile uint32_t*>(&p.ctl->changed);
      const uint32_t nit = it + 1;
      p.ctl->iter = nit;
      p.ctl->changed = 0;
      p.ctl->ctas_done = 0;
      p.ctl->converged = changed ? 0u : 1u;
      __threadfence();
      if (p.use_cond) cudaGraphSetConditional(p.cond_handle, (changed && nit < p.ctl->max_iters) ? 1u : 0u);
    }
  }
}

// ------------------------------------------------------------ init kernels
// VertexValues <- Table-3 start state (L327) or the user's initial values.
template <class A>
__global__ void init_vertex_values(const KParams p, const void* user) {
  using V_t = typename A::Value;
  V_t* vv = reinterpret_cast<V_t*>(p.vv);
  const V_t* u = reinterpret_cast<const V_t*>(user);
  for (size_t v = blockIdx.x * (size_t)blockDim.x + threadIdx.x; v < p.V; v += (size_t)gridDim.x * blockDim.x)
    vv[v] = u ? u[v] : A::start((uint32_t)v, p.source);
}

// SrcValue[e] <- VertexValues[SrcIndex[e]] for every entry (R20: a full
// write-back at t = 0), one CTA per source shard i.
template <class A>
__global__ void init_srcvalue_gs(const KParams p) {
  using V_t = typename A::Value;
  const V_t* vv = reinterpret_cast<const V_t*>(p.vv);
  const uint32_t i = blockIdx.x, lane = threadIdx.x & 31u, warp = threadIdx.x >> 5;
  gs_walk(p, i, lane, warp, blockDim.x / 32, [&](uint32_t e, uint32_t l) {
    const uint32_t u = i * p.N + l;
    p.srcvalue[e] = A::wb_value(vv[u], A::kOutDeg ? p.outdeg[u] : 0u);
  });
}
template <class A>
__global__ void init_srcvalue_cw(const KParams p) {
  using V_t = typename A::Value;
  const V_t* vv = reinterpret_cast<const V_t*>(p.vv);
  const uint32_t i = blockIdx.x, trash = p.shard_off[p.S];
  for (uint32_t k = p.cw_off[i] + threadIdx.x; k < p.cw_off[i + 1]; k += blockDim.x) {
    const uint32_t m = p.mapper[k];
    if (m == trash) continue;
    const uint32_t u = i * p.N + p.cw_src[k];
    p.srcvalue[m] = A::wb_value(vv[u], A::kOutDeg ? p.outdeg[u] : 0u);
  }
}

__global__ void reset_ctl(Ctl* ctl, uint32_t max_iters) {
  ctl->iter = 0;
  ctl->changed = 0;
  ctl->ctas_done = 0;
  ctl->max_iters = max_iters;
  ctl->converged = 0;
}

// -------------------------------------------------------------- dispatch
size_t PassKernel::smem_bytes(uint32_t N) const {
  size_t w = (size_t)words * (N + 1);
  if (wb_array) w += N;
  if (monotone) w += (N + 31) / 32;
  return ring_bytes + 4 * w;
}

template <class A, int R>
static PassKernel make_pk() {
  PassKernel k;
  k.func = reinterpret_cast<const void*>(&shard_pass<A, R>);
  k.words = A::kWords;
  k.wb_array = !A::kMonotone;
  k.monotone = A::kMonotone;
  k.ring_bytes = kStages * slot_bytes<A>();
  k.threads = kPassThreads;
  return k;
}

const PassKernel& pass_kernel(int alg, int repr) {
  static PassKernel table[kNumAlgs][2] = {
      {make_pk<AlgBFS, 0>(), make_pk<AlgBFS, 1>()},   {make_pk<AlgSSSP, 0>(), make_pk<AlgSSSP, 1>()},
      {make_pk<AlgPR, 0>(), make_pk<AlgPR, 1>()},     {make_pk<AlgCC, 0>(), make_pk<AlgCC, 1>()},
      {make_pk<AlgSSWP, 0>(), make_pk<AlgSSWP, 1>()}, {make_pk<AlgNN, 0>(), make_pk<AlgNN, 1>()},
      {make_pk<AlgHS, 0>(), make_pk<AlgHS, 1>()},     {make_pk<AlgCS, 0>(), make_pk<AlgCS, 1>()},
  };
  return table[alg][repr];
}

size_t value_bytes(int alg) { return (alg == kHS || alg == kCS) ? 8 : 4; }
bool alg_needs_edge_values(int alg) { return alg == kSSSP || alg == kSSWP || alg == kNN || alg == kHS || alg == kCS; }
bool alg_needs_init(int alg) { return alg == kNN || alg == kHS || alg == kCS; }

KParams make_params(const Graph& g, uint32_t source) {
  KParams p{};
  p.V = g.V; p.N = g.N; p.S = g.S; p.source = source;
  p.shard_off = g.d_shard_off; p.dest = g.d_dest; p.ev = g.d_ev; p.srcvalue = g.d_srcvalue;
  p.srcloc = g.d_srcloc; p.win = g.d_win; p.cw_off = g.d_cw_off; p.cw_cnt = g.d_cw_cnt;
  p.cw_src = g.d_cw_src; p.mapper = g.d_mapper; p.vv = g.d_vv; p.outdeg = g.d_outdeg;
  p.ctl = g.d_ctl; p.trace = g.d_trace; p.trace_cap = g.trace_cap;
  p.use_cond = 0; p.cond_handle = 0;
  return p;
}

template <class A>
static cudaError_t launch_init_t(const Graph& g, uint32_t source, cudaStream_t s) {
  KParams p = make_params(g, source);
  const uint32_t vb = (uint32_t)((g.V + 255) / 256);
  init_vertex_values<A><<<vb < 148 * 16 ? vb : 148 * 16, 256, 0, s>>>(p, g.d_init[A::kId]);
  if (g.S) {
    if (g.repr == CUSHA_REPR_CW) init_srcvalue_cw<A><<<g.S, 256, 0, s>>>(p);
    else init_srcvalue_gs<A><<<g.S, 256, 0, s>>>(p);
  }
  return cudaGetLastError();
}

cudaError_t launch_init(const Graph& g, int alg, uint32_t source, cudaStream_t s) {
  switch (alg) {
    case kBFS: return launch_init_t<AlgBFS>(g, source, s);
    case kSSSP: return launch_init_t<AlgSSSP>(g, source, s);
    case kPR: return launch_init_t<AlgPR>(g, source, s);
    case kCC: return launch_init_t<AlgCC>(g, source, s);
    case kSSWP: return launch_init_t<AlgSSWP>(g, source, s);
    case kNN: return launch_init_t<AlgNN>(g, source, s);
    case kHS: return launch_init_t<AlgHS>(g, source, s);
    case kCS: return launch_init_t<AlgCS>(g, source, s);
  }
  return cudaErrorInvalidValue;
}

cudaError_t launch_reset_ctl(Ctl* ctl, uint32_t max_iters, cudaStream_t s) {
  reset_ctl<<<1, 1, 0, s>>>(ctl, max_iters);
  return cudaGetLastError();
}

}  // namespace cusha
