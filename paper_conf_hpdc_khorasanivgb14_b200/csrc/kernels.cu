// kernels.cu — the shard pass (rows a1-a5) and its initialisation kernels.
//
// One launch = one CuSha iteration (Fig. 5): one CTA per shard
// (L191), four stages separated by block barriers, and the global
// convergence flag (L189, L255).  The iteration loop itself stays on the
// device: the last CTA to finish closes the iteration and sets the CUDA-graph
// while-condition, instead of the paper's
// per-iteration cudaMemcpy of is_converged (L189).
#include <cstdio>

#include "algorithms.cuh"
#include "graph.hpp"

namespace cusha {

// ----------------------------------------------------------- stage 2 body
template <class A>
__device__ __forceinline__ void proc8(uint32_t* sm, uint32_t st, const uint4& a0, const uint4& a1, const uint4& dd,
                                      const uint4& w0, const uint4& w1) {
  // 8 consecutive entries: SrcValue a0|a1, DestIndex (u16 x 8) dd, EdgeValue w0|w1
  A::compute(sm, st, dd.x & 0xFFFFu, a0.x, w0.x);
  A::compute(sm, st, dd.x >> 16, a0.y, w0.y);
  A::compute(sm, st, dd.y & 0xFFFFu, a0.z, w0.z);
  A::compute(sm, st, dd.y >> 16, a0.w, w0.w);
  A::compute(sm, st, dd.z & 0xFFFFu, a1.x, w1.x);
  A::compute(sm, st, dd.z >> 16, a1.y, w1.y);
  A::compute(sm, st, dd.w & 0xFFFFu, a1.z, w1.z);
  A::compute(sm, st, dd.w >> 16, a1.w, w1.w);
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

template <class A, int REPR>
__global__ void __launch_bounds__(kThreads) shard_pass(const KParams p) {
  extern __shared__ uint32_t sm[];
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
  if (tid == 0) { s_upd = 0; s_stores = 0; }

  // ---- stage 1: local_vertices <- init_compute(VertexValues) (Fig. 5 lines 8-10, L267)
  for (uint32_t v = tid; v < nv; v += kThreads) A::init(sm, st, v, vv[v]);
  if (tid == 0) A::init(sm, st, N, V_t{});  // trash slot for filler entries
  __syncthreads();

  // ---- stage 2: stream the shard's entries, compute() into shared memory (lines 12-13, L269)
  {
    const uint32_t cb = p.shard_off[s] >> 3, ce = p.shard_off[s + 1] >> 3;
    const uint4* sv4 = reinterpret_cast<const uint4*>(p.srcvalue);
    const uint4* d4 = reinterpret_cast<const uint4*>(p.dest);
    const uint4* e4 = reinterpret_cast<const uint4*>(p.ev);
    for (uint32_t c = cb + tid; c < ce; c += 2 * kThreads) {
      const uint32_t c2 = c + kThreads;
      const bool two = c2 < ce;
      uint4 a0 = ld_cg_v4(sv4 + 2 * (size_t)c), a1 = ld_cg_v4(sv4 + 2 * (size_t)c + 1);
      uint4 dd = ld_stream_v4(d4 + c);
      uint4 w0 = make_uint4(0, 0, 0, 0), w1 = w0, b0 = w0, b1 = w0, db = w0, x0 = w0, x1 = w0;
      if (A::kEdge) { w0 = ld_stream_v4(e4 + 2 * (size_t)c); w1 = ld_stream_v4(e4 + 2 * (size_t)c + 1); }
      if (two) {
        b0 = ld_cg_v4(sv4 + 2 * (size_t)c2); b1 = ld_cg_v4(sv4 + 2 * (size_t)c2 + 1);
        db = ld_stream_v4(d4 + c2);
        if (A::kEdge) { x0 = ld_stream_v4(e4 + 2 * (size_t)c2); x1 = ld_stream_v4(e4 + 2 * (size_t)c2 + 1); }
      }
      proc8<A>(sm, st, a0, a1, dd, w0, w1);
      if (two) proc8<A>(sm, st, b0, b1, db, x0, x1);
    }
  }
  __syncthreads();

  // ---- stage 3: update_condition, commit to VertexValues, values_updated (lines 15-20, L271)
  uint32_t my_upd = 0;
  for (uint32_t base = 0; base < nv; base += kThreads) {
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
    const uint32_t m = __ballot_sync(0xFFFFFFFFu, u);
    if (lane == 0 && m) {
      atomicAdd(&s_upd, (uint32_t)__popc(m));
    }
    if (A::kMonotone && lane == 0 && base + warp * 32 < nv) aux[(base >> 5) + warp] = m;
    my_upd |= u ? 1u : 0u;
  }
  const int any = __syncthreads_or((int)my_upd);

  // ---- stage 4: write-back into every shard's window (lines 23-26, L308)
  if (any) {
    uint32_t stores = 0;
    if (REPR == CUSHA_REPR_CW) {
      // a thread per CW_s entry: SrcValue[Mapper[k]] = local[SrcIndex[k]] (L177, Fig. 4b)
      const uint32_t kb = p.cw_off[s] >> 3, ke = p.cw_off[s + 1] >> 3;
      const uint4* c4 = reinterpret_cast<const uint4*>(p.cw_src);
      const uint4* m4 = reinterpret_cast<const uint4*>(p.mapper);
      const uint32_t trash = p.shard_off[p.S];
      for (uint32_t c = kb + tid; c < ke; c += kThreads) {
        const uint4 ii = ld_stream_v4(c4 + c);
        const uint4 m0 = ld_stream_v4(m4 + 2 * (size_t)c), m1 = ld_stream_v4(m4 + 2 * (size_t)c + 1);
        const uint32_t L[8] = {ii.x & 0xFFFFu, ii.x >> 16, ii.y & 0xFFFFu, ii.y >> 16,
                               ii.z & 0xFFFFu, ii.z >> 16, ii.w & 0xFFFFu, ii.w >> 16};
        const uint32_t M[8] = {m0.x, m0.y, m0.z, m0.w, m1.x, m1.y, m1.z, m1.w};
#pragma unroll
        for (int k = 0; k < 8; ++k) {
          uint32_t val;
          if (M[k] != trash && wb_get<A>(sm, aux, L[k], val)) { st_u32(p.srcvalue + M[k], val); ++stores; }
        }
      }
    } else {
      // G-Shards: one warp per target shard j iterates W_sj (L151, Fig. 3c)
      const uint32_t* r0 = p.win + (size_t)s * p.S;
      const uint32_t* r1 = r0 + p.S;
      for (uint32_t jb = warp * 32; jb < p.S; jb += kThreads) {
        const uint32_t j = jb + lane;
        uint32_t a = 0, b = 0;
        if (j < p.S) { a = __ldg(r0 + j); b = __ldg(r1 + j); }
        uint32_t todo = __ballot_sync(0xFFFFFFFFu, b > a);
        while (todo) {
          const int k = __ffs(todo) - 1;
          todo &= todo - 1;
          const uint32_t wa = __shfl_sync(0xFFFFFFFFu, a, k), we = __shfl_sync(0xFFFFFFFFu, b, k);
          for (uint32_t e = wa + lane; e < we; e += 32) {
            const uint32_t l = __ldg(p.srcidx + e) - off;
            uint32_t val;
            if (wb_get<A>(sm, aux, l, val)) { st_u32(p.srcvalue + e, val); ++stores; }
          }
        }
      }
    }
    for (int o = 16; o; o >>= 1) stores += __shfl_xor_sync(0xFFFFFFFFu, stores, o);
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

// SrcValue[e] <- VertexValues[SrcIndex[e]] for every entry (R20: a full write-back at t = 0).
template <class A>
__global__ void init_srcvalue_gs(const KParams p, uint64_t P) {
  using V_t = typename A::Value;
  const V_t* vv = reinterpret_cast<const V_t*>(p.vv);
  for (size_t e = blockIdx.x * (size_t)blockDim.x + threadIdx.x; e < P; e += (size_t)gridDim.x * blockDim.x) {
    if (p.dest[e] == p.N) continue;  // filler
    const uint32_t u = p.srcidx[e];
    p.srcvalue[e] = A::wb_value(vv[u], A::kOutDeg ? p.outdeg[u] : 0u);
  }
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
  return 4 * w;
}

template <class A, int R>
static PassKernel make_pk() {
  PassKernel k;
  k.func = reinterpret_cast<const void*>(&shard_pass<A, R>);
  k.words = A::kWords;
  k.wb_array = !A::kMonotone;
  k.monotone = A::kMonotone;
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
  p.srcidx = g.d_srcidx; p.win = g.d_win; p.cw_off = g.d_cw_off; p.cw_cnt = g.d_cw_cnt;
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
  if (g.repr == CUSHA_REPR_CW) {
    if (g.S) init_srcvalue_cw<A><<<g.S, 256, 0, s>>>(p);
  } else {
    const uint64_t eb = (g.P + 255) / 256;
    if (g.P) init_srcvalue_gs<A><<<(unsigned)(eb < 148 * 32 ? eb : 148 * 32), 256, 0, s>>>(p, g.P);
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
