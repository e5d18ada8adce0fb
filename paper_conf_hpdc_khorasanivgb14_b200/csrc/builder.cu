// builder.cu — row a0: G-Shards and Concatenated Windows built on the device.
//
// PAPER.md §3.1 L119-155 (G-Shards: Partitioned L128, Ordered L129, windows
// W_ij L155) and §3.2 L175-179 (CW_i = SrcIndex of W_i0..W_i(p-1) in j order,
// Mapper).  The paper builds on the host and copies the result over PCIe
// (L457); here the edge list is copied once (12 B/edge) and the layout is
// produced in HBM by radix sorts (CUB, a library primitive used at setup time
// only) and a few scatter kernels.
//
// G-Shards order = lexicographic (shard(dst), src, dst, input index): one
// stable radix sort of the packed key (shard(dst) | src | dst mod N) — the
// input index tie-break (R17) comes from the sort's stability.  CW needs no
// second sort: CW_i is by definition W_i0, W_i1, ..., W_i(S-1) concatenated
// (L175), and each W_ij is the contiguous range [win[i][j], win[i+1][j]) of
// shard j (L155), so Mapper and SrcIndexCW are read off the window table.
#include <cub/cub.cuh>

#include <algorithm>
#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <string>
#include <vector>

#include "common.cuh"
#include "graph.hpp"

namespace cusha {

namespace {

int bits_for(uint64_t maxval) {  // bits needed to represent 0..maxval
  int b = 0;
  while (b < 64 && (1ull << b) <= maxval) ++b;
  return b;
}

inline unsigned grid_for(uint64_t n, unsigned block = 256) {
  uint64_t g = (n + block - 1) / block;
  const uint64_t cap = 148ull * 64;
  if (g > cap) g = cap;
  return (unsigned)(g ? g : 1);
}

#define GRID_STRIDE(i, n) for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < (n); i += (uint64_t)gridDim.x * blockDim.x)

// One pass over the input edges [lo, hi): the G-Shards sort key, the input
// index (the sort's payload, R17), out-degrees (PR NbrsNum, L318) and
// in-degrees (fixed-point range check).  Run per chunk as the host copy
// streams in (DESIGN.md f2).
__global__ void k_ingest(const uint32_t* __restrict__ src, const uint32_t* __restrict__ dst, uint64_t lo, uint64_t hi,
                         uint32_t V, uint32_t N, int bn, int bsrc, uint64_t* keys, uint32_t* ids, uint32_t* bad,
                         uint32_t* outdeg, uint32_t* indeg) {
  GRID_STRIDE(i, hi - lo) {
    const uint64_t e = lo + i;
    const uint32_t s = src[e], d = dst[e];
    if (s >= V || d >= V) {
      *bad = 1;
      keys[e] = 0;
    } else {
      keys[e] = ((uint64_t)(d / N) << (bsrc + bn)) | ((uint64_t)s << bn) | (uint64_t)(d % N);
      atomicAdd(&outdeg[s], 1u);
      if (indeg) atomicAdd(&indeg[d], 1u);
    }
    ids[e] = (uint32_t)e;
  }
}

// ---- chunked G-Shards sort (row f2).  With a host edge list
// each input chunk is radix-sorted as soon as its copy lands and folded into
// the sorted prefix of the earlier chunks by a stable merge: on equal keys the
// prefix goes first, and every input index in it is smaller, so the result is
// the one stable sort of the whole list (R17).  Only the last chunk's sort and
// one merge pass remain after the copy.
constexpr int kMergeItems = 8, kMergeThreads = 256, kMergeTile = kMergeItems * kMergeThreads;

// merge path: how many of the first d outputs come from a (ties: a first)
template <class I>
__device__ __forceinline__ I merge_split(const uint64_t* a, I na, const uint64_t* b, I nb, I d) {
  I lo = d > nb ? d - nb : 0, hi = d < na ? d : na;
  while (lo < hi) {
    const I mid = (lo + hi) >> 1;
    if (a[mid] <= b[d - mid - 1]) lo = mid + 1;
    else hi = mid;
  }
  return lo;
}
__global__ void k_merge_splits(const uint64_t* __restrict__ a, uint64_t na, const uint64_t* __restrict__ b, uint64_t nb,
                               uint64_t tiles, uint64_t* split) {
  GRID_STRIDE(t, tiles + 1) split[t] = merge_split<uint64_t>(a, na, b, nb, min(t * (uint64_t)kMergeTile, na + nb));
}
// one tile of kMergeTile outputs per block: both input ranges staged in shared
// memory, kMergeItems outputs per thread, written back coalesced
__global__ void __launch_bounds__(kMergeThreads) k_merge(const uint64_t* __restrict__ ak, const uint32_t* __restrict__ ai,
                                                         uint64_t na, const uint64_t* __restrict__ bk,
                                                         const uint32_t* __restrict__ bi, uint64_t nb,
                                                         const uint64_t* __restrict__ split, uint64_t* ok, uint32_t* oi) {
  __shared__ uint64_t sk[kMergeTile];
  __shared__ uint32_t si[kMergeTile];
  const uint64_t d0 = blockIdx.x * (uint64_t)kMergeTile, d1 = min(d0 + kMergeTile, na + nb);
  const uint64_t a0 = split[blockIdx.x], a1 = split[blockIdx.x + 1], b0 = d0 - a0;
  const uint32_t la = (uint32_t)(a1 - a0), n = (uint32_t)(d1 - d0), lb = n - la;
  for (uint32_t x = threadIdx.x; x < n; x += kMergeThreads) {
    if (x < la) { sk[x] = ak[a0 + x]; si[x] = ai[a0 + x]; }
    else { sk[x] = bk[b0 + x - la]; si[x] = bi[b0 + x - la]; }
  }
  __syncthreads();
  const uint32_t d = min((uint32_t)threadIdx.x * kMergeItems, n);
  uint32_t i = merge_split<uint32_t>(sk, la, sk + la, lb, d), j = d - i;
  uint64_t rk[kMergeItems];
  uint32_t ri[kMergeItems];
#pragma unroll
  for (int k = 0; k < kMergeItems; ++k) {
    if (d + k < n) {
      const bool from_a = j >= lb || (i < la && sk[i] <= sk[la + j]);
      const uint32_t x = from_a ? i++ : la + j++;
      rk[k] = sk[x];
      ri[k] = si[x];
    }
  }
  __syncthreads();
#pragma unroll
  for (int k = 0; k < kMergeItems; ++k)
    if (d + k < n) { sk[d + k] = rk[k]; si[d + k] = ri[k]; }
  __syncthreads();
  for (uint32_t x = threadIdx.x; x < n; x += kMergeThreads) {
    ok[d0 + x] = sk[x];
    oi[d0 + x] = si[x];
  }
}

// largest in-degree (fixed-point range check) from the shards: in-edges of a
// vertex all sit in its shard, so one block per shard counts its DestIndex
// values in shared memory (N counters) — no global atomics during ingest
__global__ void k_indeg_max(const uint16_t* __restrict__ dest, const uint32_t* __restrict__ off,
                            const uint32_t* __restrict__ cnt, uint32_t N, uint32_t* out) {
  extern __shared__ uint32_t hist[];
  for (uint32_t v = threadIdx.x; v < N; v += blockDim.x) hist[v] = 0;
  __syncthreads();
  const uint32_t b = off[blockIdx.x], e = b + cnt[blockIdx.x];
  for (uint32_t p = b + threadIdx.x; p < e; p += blockDim.x) atomicAdd(&hist[dest[p]], 1u);
  __syncthreads();
  uint32_t m = 0;
  for (uint32_t v = threadIdx.x; v < N; v += blockDim.x) m = max(m, hist[v]);
  for (int o = 16; o; o >>= 1) m = max(m, __shfl_xor_sync(0xFFFFFFFFu, m, o));
  if ((threadIdx.x & 31) == 0 && m) atomicMax(out, m);
}

// start[t] = first sorted index whose (key >> shift) >= t, for t = 0..S
__global__ void k_starts(const uint64_t* __restrict__ k, uint64_t E, int shift, uint64_t mask, uint32_t S,
                         uint32_t* start) {
  GRID_STRIDE(p, E + 1) {
    const int64_t cur = p < E ? (int64_t)((k[p] >> shift) & mask) : (int64_t)S;
    const int64_t prev = p == 0 ? -1 : (int64_t)((k[p - 1] >> shift) & mask);
    for (int64_t t = prev + 1; t <= cur; ++t) start[t] = (uint32_t)p;
  }
}
// cnt[s] = start[s+1]-start[s]; padded[s] = round up to kPad; padded[S] = 0
__global__ void k_counts(const uint32_t* start, uint32_t S, uint32_t* cnt, uint64_t* padded) {
  GRID_STRIDE(s, (uint64_t)S + 1) {
    if (s < S) {
      const uint32_t c = start[s + 1] - start[s];
      cnt[s] = c;
      padded[s] = (uint64_t)((c + kPad - 1) / kPad) * kPad;
    } else {
      padded[s] = 0;
    }
  }
}
__global__ void k_narrow(const uint64_t* in, uint64_t n, uint32_t* out) {
  GRID_STRIDE(i, n) out[i] = (uint32_t)in[i];
}

// filler entries of every shard: DestIndex = N (trash slot), no edge
__global__ void k_fill_shard_pads(const uint32_t* off, const uint32_t* cnt, uint32_t S, uint32_t N, uint16_t* dest,
                                  uint16_t* srcidx, uint32_t* eid, uint32_t* ev) {
  GRID_STRIDE(i, (uint64_t)S * kPad) {
    const uint32_t s = (uint32_t)(i / kPad), r = (uint32_t)(i % kPad);
    const uint32_t pos = off[s] + cnt[s] + r;
    if (pos < off[s + 1]) {
      dest[pos] = (uint16_t)N;
      srcidx[pos] = 0;
      if (eid) eid[pos] = 0xFFFFFFFFu;
      if (ev) ev[pos] = 0;
    }
  }
}

__global__ void k_scatter_gs(const uint64_t* __restrict__ keys, const uint32_t* __restrict__ ids, uint64_t E,
                             const uint32_t* start, const uint32_t* off, int bn, int bsrc, const uint32_t* __restrict__ val,
                             uint32_t N, uint16_t* dest, uint16_t* srcidx, uint32_t* eid, uint32_t* ev) {
  const uint64_t mn = (1ull << bn) - 1, ms = (1ull << bsrc) - 1;
  GRID_STRIDE(p, E) {
    const uint64_t k = keys[p];
    const uint32_t sh = (uint32_t)(k >> (bsrc + bn));
    const uint32_t pp = off[sh] + (uint32_t)(p - start[sh]);
    dest[pp] = (uint16_t)(k & mn);
    srcidx[pp] = (uint16_t)(((k >> bn) & ms) % N);  // SrcIndex local to its source shard
    const uint32_t id = ids[p];
    if (eid) eid[pp] = id;
    if (ev) ev[pp] = val[id];
  }
}

// window table: win[t*S + j] = first padded position of shard j with SrcIndex >= t*N (t = 0..S)
__global__ void k_windows(const uint64_t* __restrict__ keys, uint64_t E, const uint32_t* start, const uint32_t* off,
                          uint32_t N, uint32_t S, int bn, int bsrc, uint32_t* win) {
  const uint64_t ms = (1ull << bsrc) - 1;
  GRID_STRIDE(p, E) {
    const uint64_t k = keys[p];
    const uint32_t j = (uint32_t)(k >> (bsrc + bn));
    const int64_t i = (int64_t)(((k >> bn) & ms) / N);
    const int64_t pi = (p == start[j]) ? -1 : (int64_t)(((keys[p - 1] >> bn) & ms) / N);
    const uint32_t pos = off[j] + (uint32_t)(p - start[j]);  // shard position of sorted entry p
    for (int64_t t = pi + 1; t <= i; ++t) win[(size_t)t * S + j] = pos;
  }
}
__global__ void k_windows_tail(const uint64_t* __restrict__ keys, const uint32_t* start, const uint32_t* off,
                               const uint32_t* cnt, uint32_t N, uint32_t S, int bn, int bsrc, uint32_t* win) {
  const uint64_t ms = (1ull << bsrc) - 1;
  GRID_STRIDE(j, (uint64_t)S) {
    int64_t last = -1;
    if (cnt[j]) last = (int64_t)(((keys[start[j + 1] - 1] >> bn) & ms) / N);
    const uint32_t end = off[j] + cnt[j];
    for (int64_t t = last + 1; t <= (int64_t)S; ++t) win[(size_t)t * S + j] = end;
  }
}

__global__ void k_max_u32(const uint32_t* __restrict__ a, uint64_t n, uint32_t* out) {
  uint32_t m = 0;
  GRID_STRIDE(i, n) m = max(m, a[i]);
  for (int o = 16; o; o >>= 1) m = max(m, __shfl_xor_sync(0xFFFFFFFFu, m, o));
  if ((threadIdx.x & 31) == 0 && m) atomicMax(out, m);
}
// largest |x| of raw 4-byte values read as f32 (non-finite: +inf bits)
__global__ void k_max_abs_f32(const uint32_t* __restrict__ a, uint64_t n, uint32_t* out) {
  uint32_t m = 0;
  GRID_STRIDE(i, n) {
    uint32_t b = a[i] & 0x7FFFFFFFu;
    if (b > 0x7F800000u) b = 0x7F800000u;  // NaN counts as infinite
    m = max(m, b);                          // non-negative floats order like their bits
  }
  for (int o = 16; o; o >>= 1) m = max(m, __shfl_xor_sync(0xFFFFFFFFu, m, o));
  if ((threadIdx.x & 31) == 0 && m) atomicMax(out, m);
}

// |CW_i| = sum of out-degrees over shard i's vertex range
__global__ void k_cw_counts(const uint32_t* outdeg, uint32_t V, uint32_t N, uint32_t* cw_cnt) {
  const uint32_t i = blockIdx.x;
  const uint32_t b = i * N, e = min(V, b + N);
  uint32_t acc = 0;
  for (uint32_t v = b + threadIdx.x; v < e; v += blockDim.x) acc += outdeg[v];
  typedef cub::BlockReduce<uint32_t, 256> BR;
  __shared__ typename BR::TempStorage tmp;
  acc = BR(tmp).Sum(acc);
  if (threadIdx.x == 0) cw_cnt[i] = acc;
}

// padded[i] = cnt[i] rounded up to kPad; padded[S] = 0 (exclusive scan input)
__global__ void k_pad_counts(const uint32_t* cnt, uint32_t S, uint64_t* padded) {
  GRID_STRIDE(i, (uint64_t)S + 1) padded[i] = i < S ? (uint64_t)((cnt[i] + kPad - 1) / kPad) * kPad : 0ull;
}

// CW_i from the window table (L175, Fig. 4a): block i walks row i of the
// table 256 windows at a time; a block scan of the window lengths gives each
// window's offset inside CW_i, and the block's threads then copy the chunk's
// entries (one per thread, the window found by binary search over the
// chunk's offsets): Mapper[k] = shard position, SrcIndexCW[k] = SrcIndex there.
__global__ void __launch_bounds__(256) k_cw_from_windows(const uint32_t* __restrict__ win, uint32_t S,
                                                         const uint32_t* __restrict__ cw_off,
                                                         const uint16_t* __restrict__ srcidx, uint16_t* cw_src,
                                                         uint32_t* mapper, uint16_t* cw_win, uint32_t* cw_delta) {
  typedef cub::BlockScan<uint32_t, 256> BS;
  __shared__ typename BS::TempStorage tmp;
  __shared__ uint32_t s_off[257], s_beg[256];
  const uint32_t i = blockIdx.x, tid = threadIdx.x;
  const uint32_t* r0 = win + (size_t)i * S;
  const uint32_t* r1 = r0 + S;
  uint32_t base = cw_off[i];
  for (uint32_t j0 = 0; j0 < S; j0 += 256) {
    const uint32_t j = j0 + tid;
    uint32_t b = 0, len = 0;
    if (j < S) { b = r0[j]; len = r1[j] - b; }
    uint32_t ex, total;
    BS(tmp).ExclusiveSum(len, ex, total);
    s_off[tid] = ex;
    s_beg[tid] = b;
    if (tid == 0) s_off[256] = total;
    // Mapper in window form: W_ij's entries sit at CW positions base+ex.. and
    // shard positions b.., so Mapper[k] = (b - (base + ex)) + k (mod 2^32)
    if (j < S) cw_delta[(size_t)i * S + j] = b - (base + ex);
    __syncthreads();
    for (uint32_t f = tid; f < total; f += 256) {
      uint32_t lo = 0, hi = 256;  // last window w with s_off[w] <= f
      while (hi - lo > 1) {
        const uint32_t mid = (lo + hi) >> 1;
        if (s_off[mid] <= f) lo = mid;
        else hi = mid;
      }
      const uint32_t pos = s_beg[lo] + (f - s_off[lo]);
      mapper[base + f] = pos;
      cw_win[base + f] = (uint16_t)(j0 + lo);
      cw_src[base + f] = srcidx[pos];  // SrcIndex - i*N
    }
    base += total;
    __syncthreads();
  }
}
__global__ void k_fill_cw_pads(const uint32_t* coff, const uint32_t* ccnt, uint32_t S, uint32_t trash, uint16_t* cw_src,
                               uint32_t* mapper, uint16_t* cw_win) {
  GRID_STRIDE(i, (uint64_t)S * kPad) {
    const uint32_t s = (uint32_t)(i / kPad), r = (uint32_t)(i % kPad);
    const uint32_t pos = coff[s] + ccnt[s] + r;
    if (pos < coff[s + 1]) {
      cw_src[pos] = 0;
      mapper[pos] = trash;
      cw_win[pos] = 0xFFFFu;
    }
  }
}

// Build temporaries are stream-ordered allocations on the graph's stream
// (cudaMallocAsync from the device pool, which cusha_build_graph sets to
// retain freed memory): repeated builds neither map nor unmap HBM.
thread_local cudaStream_t t_alloc_stream = nullptr;
struct DevBuf {  // RAII temporary
  void* p = nullptr;
  ~DevBuf() { if (p) cudaFreeAsync(p, t_alloc_stream); }
};

// Diagnostics only: CUSHA_DEBUG_BUILD=1 prints the wall time of each build
// phase (synchronising at every mark, so it perturbs what it measures).
struct PhaseTimer {
  bool on = std::getenv("CUSHA_DEBUG_BUILD") != nullptr;
  cudaStream_t st;
  std::chrono::steady_clock::time_point t = std::chrono::steady_clock::now();
  explicit PhaseTimer(cudaStream_t s) : st(s) {}
  void mark(const char* what) {
    if (!on) return;
    cudaStreamSynchronize(st);
    const auto n = std::chrono::steady_clock::now();
    std::fprintf(stderr, "[cusha build] %-28s %9.3f ms\n", what,
                 std::chrono::duration<double, std::milli>(n - t).count());
    t = n;
  }
};

#define CK(call)                                                                     \
  do {                                                                               \
    cudaError_t e_ = (call);                                                         \
    if (e_ != cudaSuccess) {                                                         \
      err = std::string(#call) + ": " + cudaGetErrorString(e_);                      \
      return e_ == cudaErrorMemoryAllocation ? CUSHA_ENOMEM : CUSHA_ECUDA;           \
    }                                                                                \
  } while (0)

template <class T>
cudaError_t dalloc(T** p, uint64_t n) {
  return dev_alloc(reinterpret_cast<void**>(p), (n ? n : 1) * sizeof(T), t_alloc_stream);
}

// ---- run-length form of Mapper
// Within a window W_ij the Mapper targets of CW_i are consecutive shard
// positions (CW_i lists W_ij in shard order, L175, and W_ij is contiguous in
// shard j, L155), so Mapper is a run per non-empty window:
//   RunK[r] = CW position of the run's first entry, RunT[r] = its target.
// RunUnit[u] = last run with RunK <= u*kRunUnit (locates a tile's runs).
__global__ void k_win_len(const uint32_t* __restrict__ win, uint32_t S, uint32_t* len, uint32_t* nonempty) {
  GRID_STRIDE(t, (uint64_t)S * S) {
    const uint32_t l = win[t + S] - win[t];  // row i = t / S, column j
    len[t] = l;
    nonempty[t] = l ? 1u : 0u;
  }
}
__global__ void k_runs(const uint32_t* __restrict__ win, const uint32_t* len, const uint32_t* pos, const uint32_t* ridx,
                       const uint32_t* cw_off, uint32_t S, uint32_t* run_k, uint32_t* run_t) {
  GRID_STRIDE(t, (uint64_t)S * S) {
    if (!len[t]) continue;
    const uint32_t i = (uint32_t)(t / S);
    const uint32_t r = ridx[t];
    run_k[r] = cw_off[i] + (pos[t] - pos[(size_t)i * S]);
    run_t[r] = win[t];
  }
}
__global__ void k_run_pad(uint32_t R, uint32_t Rpad, uint32_t* run_k, uint32_t* run_t) {
  GRID_STRIDE(r, (uint64_t)Rpad) {
    if (r >= R) { run_k[r] = 0xFFFFFFFFu; run_t[r] = 0; }
  }
}
__global__ void k_run_delta(const uint32_t* run_k, const uint32_t* run_t, uint64_t n, uint32_t* run_d) {
  GRID_STRIDE(r, n) run_d[r] = run_t[r] - run_k[r];
}
__global__ void k_run_bits(const uint32_t* __restrict__ run_k, uint32_t R, uint32_t* bits) {
  GRID_STRIDE(r, (uint64_t)R) atomicOr(&bits[run_k[r] >> 5], 1u << (run_k[r] & 31));
}
__global__ void k_run_unit(const uint32_t* __restrict__ run_k, uint32_t R, uint64_t U, uint32_t* unit) {
  GRID_STRIDE(u, U) {
    const uint64_t pos = u * kRunUnit;
    uint32_t lo = 0, hi = R;  // first run with run_k > pos
    while (lo < hi) {
      const uint32_t mid = (lo + hi) >> 1;
      if ((uint64_t)run_k[mid] <= pos) lo = mid + 1;
      else hi = mid;
    }
    unit[u] = lo ? lo - 1 : 0;
  }
}

}  // namespace

int build_runs(Graph& g, std::string& err) {
  cudaStream_t st = g.stream;
  t_alloc_stream = st;
  const uint32_t S = g.S;
  const uint64_t S2 = (uint64_t)S * S;
  DevBuf len, nonempty, pos, ridx, t1, t2;
  CK(dalloc((uint32_t**)&len.p, S2));
  CK(dalloc((uint32_t**)&nonempty.p, S2));
  CK(dalloc((uint32_t**)&pos.p, S2));
  CK(dalloc((uint32_t**)&ridx.p, S2 + 1));
  k_win_len<<<grid_for(S2), 256, 0, st>>>(g.d_win, S, (uint32_t*)len.p, (uint32_t*)nonempty.p);
  CK(cudaGetLastError());
  size_t b1 = 0, b2 = 0;
  CK(cub::DeviceScan::ExclusiveSum(nullptr, b1, (uint32_t*)len.p, (uint32_t*)pos.p, (int64_t)S2, st));
  CK(dev_alloc(&t1.p, b1 ? b1 : 1, st));
  CK(cub::DeviceScan::ExclusiveSum(t1.p, b1, (uint32_t*)len.p, (uint32_t*)pos.p, (int64_t)S2, st));
  CK(cub::DeviceScan::InclusiveSum(nullptr, b2, (uint32_t*)nonempty.p, (uint32_t*)ridx.p + 1, (int64_t)S2, st));
  CK(dev_alloc(&t2.p, b2 ? b2 : 1, st));
  CK(cudaMemsetAsync(ridx.p, 0, 4, st));
  CK(cub::DeviceScan::InclusiveSum(t2.p, b2, (uint32_t*)nonempty.p, (uint32_t*)ridx.p + 1, (int64_t)S2, st));
  uint32_t R = 0;
  CK(cudaMemcpyAsync(&R, (uint32_t*)ridx.p + S2, 4, cudaMemcpyDeviceToHost, st));
  CK(cudaStreamSynchronize(st));
  g.R = R;
  const uint64_t Rpad = ((uint64_t)R + 3) / 4 * 4 + 8;  // TMA copies round run ranges to 4 (16 B)
  CK(dalloc(&g.d_run_k, Rpad));
  CK(dalloc(&g.d_run_t, Rpad));
  k_run_pad<<<grid_for(Rpad), 256, 0, st>>>(R, (uint32_t)Rpad, g.d_run_k, g.d_run_t);
  k_runs<<<grid_for(S2), 256, 0, st>>>(g.d_win, (uint32_t*)len.p, (uint32_t*)pos.p, (uint32_t*)ridx.p, g.d_cw_off, S,
                                       g.d_run_k, g.d_run_t);
  const uint64_t U = g.Q / kRunUnit + 2;
  CK(dalloc(&g.d_run_unit, U + 4));  // + 4: 16-byte TMA slices rounded up
  k_run_unit<<<grid_for(U), 256, 0, st>>>(g.d_run_k, R, U, g.d_run_unit);
  const uint64_t W = g.Q / 32 + 16;  // run-start bitmap (+ slack for 128-entry aligned TMA slices)
  CK(dalloc(&g.d_run_bits, W));
  CK(cudaMemsetAsync(g.d_run_bits, 0, W * 4, st));
  k_run_bits<<<grid_for(R), 256, 0, st>>>(g.d_run_k, R, g.d_run_bits);
  CK(dalloc(&g.d_run_d, Rpad));
  k_run_delta<<<grid_for(Rpad), 256, 0, st>>>(g.d_run_k, g.d_run_t, Rpad, g.d_run_d);
  CK(cudaGetLastError());
  CK(cudaStreamSynchronize(st));
  return CUSHA_OK;
}

int build_layout(Graph& g, const uint32_t* d_src, const uint32_t* d_dst, const uint32_t* d_val, std::string& err,
                 const InputChunks* chunks) {
  cudaStream_t st = g.stream;
  const uint64_t E = g.E;
  const uint32_t V = g.V, N = g.N, S = g.S;
  g.s0 = 0; g.Sl = S; g.v0 = 0; g.nvl = V; g.E_loc = E;
  const int bn = bits_for(N - 1) ? bits_for(N - 1) : 1, bsrc = bits_for(V - 1) ? bits_for(V - 1) : 1,
            bsh = bits_for(S - 1);
  const int total = bsh + bsrc + bn;
  if (total > 64) { err = "key does not fit 64 bits"; return CUSHA_EINVAL; }
  PhaseTimer pt(st);
  t_alloc_stream = st;

  DevBuf bad, start, padded, temp, indeg, mx;
  // the sort's key / index buffers are views into one slab: one request of the
  // same size per build, which the pool meets with the block the previous
  // build freed (separate requests fragmented it, and a build that found no
  // block to fit mapped new memory: 80-95 ms instead of 0.1 ms)
  struct View {
    void* p = nullptr;
  };
  DevBuf slab;
  View keys, keys2, ids, ids2;
  // per-chunk sorts + merges (host input in several chunks) when the third
  // pair of key/index buffers fits comfortably; otherwise one sort at the end
  // (same result, DESIGN.md f2)
  const int nch = chunks && chunks->n ? chunks->n : 1;
  bool chunk_sort = nch > 1 && E && !std::getenv("CUSHA_NO_CHUNK_SORT");
  if (chunk_sort) {
    size_t fr = 0, tot = 0;
    chunk_sort = cudaMemGetInfo(&fr, &tot) == cudaSuccess && fr > 48 * E + (2ull << 30);
  }
  View keys3, ids3, splits;
  {
    const uint64_t e1 = E ? E : 1;
    auto al = [](uint64_t b) { return (b + 255) & ~255ull; };
    uint64_t off[7] = {}, at = 0;
    const uint64_t sz[7] = {8 * e1, 8 * e1, 4 * e1, 4 * e1, chunk_sort ? 8 * e1 : 0, chunk_sort ? 4 * e1 : 0,
                            chunk_sort ? 8 * (E / kMergeTile + 2) : 0};
    for (int i = 0; i < 7; ++i) { off[i] = at; at += al(sz[i]); }
    CK(dev_alloc(&slab.p, at, t_alloc_stream));
    uint8_t* b = static_cast<uint8_t*>(slab.p);
    View* v[7] = {&keys, &keys2, &ids, &ids2, &keys3, &ids3, &splits};
    for (int i = 0; i < 7; ++i) v[i]->p = sz[i] ? b + off[i] : nullptr;
  }
  uint64_t max_chunk = 0;
  if (chunk_sort) {
    for (int c = 0; c < nch; ++c) max_chunk = std::max(max_chunk, chunks->bounds[c + 1] - chunks->bounds[c]);
    size_t tb = 0;
    cub::DoubleBuffer<uint64_t> kq(nullptr, nullptr);
    cub::DoubleBuffer<uint32_t> vq(nullptr, nullptr);
    CK(cub::DeviceRadixSort::SortPairs(nullptr, tb, kq, vq, (int64_t)max_chunk, 0, total, st));
    CK(dev_alloc(&temp.p, tb ? tb : 1, st));
  }
  CK(dalloc(&g.d_outdeg, V));
  // in-degrees: counted per shard after the scatter when N counters fit in
  // shared memory, else by global atomics during ingest
  const bool hist_indeg = 4ull * N <= 96 * 1024;
  if (!hist_indeg) CK(dalloc((uint32_t**)&indeg.p, V));
  CK(dalloc((uint32_t**)&mx.p, 2));
  pt.mark("alloc keys/ids");
  CK(dalloc((uint32_t**)&bad.p, 1));
  CK(cudaMemsetAsync(bad.p, 0, 4, st));
  CK(cudaMemsetAsync(g.d_outdeg, 0, (size_t)V * 4, st));
  if (!hist_indeg) CK(cudaMemsetAsync(indeg.p, 0, (size_t)V * 4, st));
  CK(cudaMemsetAsync(mx.p, 0, 8, st));
  // keys + degrees per input chunk, each as soon as its host copy has landed
  // chunked sort: raw chunk c lands in (keys, ids)[lo, hi); it is sorted with
  // (keys2, ids2)[lo, hi) as the alternate buffer — free, since the sorted
  // prefix occupies [0, lo) of whichever of (keys2, ids2) / (keys3, ids3) holds
  // it — and merged with the prefix into the other one.
  uint64_t* pk = (uint64_t*)keys2.p;
  uint32_t* pi = (uint32_t*)ids2.p;
  uint64_t* qk = (uint64_t*)keys3.p;
  uint32_t* qi = (uint32_t*)ids3.p;
  for (int c = 0; c < nch; ++c) {
    const uint64_t lo = chunks && chunks->n ? chunks->bounds[c] : 0, hi = chunks && chunks->n ? chunks->bounds[c + 1] : E;
    if (chunks && chunks->n) CK(cudaStreamWaitEvent(st, chunks->ready[c], 0));
    if (hi > lo)
      k_ingest<<<grid_for(hi - lo), 256, 0, st>>>(d_src, d_dst, lo, hi, V, N, bn, bsrc, (uint64_t*)keys.p,
                                                  (uint32_t*)ids.p, (uint32_t*)bad.p, g.d_outdeg, (uint32_t*)indeg.p);
    if (chunk_sort) {
      const uint64_t n = hi - lo;
      cub::DoubleBuffer<uint64_t> kq((uint64_t*)keys.p + lo, pk + lo);
      cub::DoubleBuffer<uint32_t> vq((uint32_t*)ids.p + lo, pi + lo);
      size_t tb = 0;
      CK(cub::DeviceRadixSort::SortPairs(nullptr, tb, kq, vq, (int64_t)max_chunk, 0, total, st));
      if (n) CK(cub::DeviceRadixSort::SortPairs(temp.p, tb, kq, vq, (int64_t)n, 0, total, st));
      const uint64_t tiles = (hi + kMergeTile - 1) / kMergeTile;
      k_merge_splits<<<grid_for(tiles + 1), 256, 0, st>>>(pk, lo, kq.Current(), n, tiles, (uint64_t*)splits.p);
      if (tiles)
        k_merge<<<(unsigned)tiles, kMergeThreads, 0, st>>>(pk, pi, lo, kq.Current(), vq.Current(), n,
                                                            (uint64_t*)splits.p, qk, qi);
      std::swap(pk, qk);
      std::swap(pi, qi);
    }
  }
  CK(cudaGetLastError());
  // range of the float algorithms' fixed-point sums (include/cusha.h "Fixed-point range")
  if (!hist_indeg) k_max_u32<<<grid_for(V), 256, 0, st>>>((uint32_t*)indeg.p, V, (uint32_t*)mx.p);
  // h and ev_bits receive async copies: the guard drains the stream before they go
  uint32_t h[2] = {0, 0}, ev_bits = 0;
  struct DrainOnExit {
    cudaStream_t s;
    ~DrainOnExit() { cudaStreamSynchronize(s); }
  } drain{st};
  CK(cudaMemcpyAsync(h + 1, bad.p, 4, cudaMemcpyDeviceToHost, st));
  CK(cudaStreamSynchronize(st));
  if (h[1]) { err = "edge endpoint >= num_vertices"; return CUSHA_EINVAL; }
  pt.mark("keys + degrees + validate");

  // ---- G-Shards order
  cub::DoubleBuffer<uint64_t> kb((uint64_t*)keys.p, (uint64_t*)keys2.p);
  cub::DoubleBuffer<uint32_t> vb((uint32_t*)ids.p, (uint32_t*)ids2.p);
  size_t tbytes = 0;
  if (E && !chunk_sort) {
    CK(cub::DeviceRadixSort::SortPairs(nullptr, tbytes, kb, vb, (int64_t)E, 0, total, st));
    CK(dev_alloc(&temp.p, tbytes, st));
    CK(cub::DeviceRadixSort::SortPairs(temp.p, tbytes, kb, vb, (int64_t)E, 0, total, st));
  }
  pt.mark("G-Shards sort");
  const uint64_t* K = chunk_sort ? pk : kb.Current();
  const uint32_t* I = chunk_sort ? pi : vb.Current();

  CK(dalloc((uint32_t**)&start.p, (uint64_t)S + 1));
  CK(dalloc((uint64_t**)&padded.p, (uint64_t)S + 1));
  CK(dalloc(&g.d_shard_cnt, S));
  CK(dalloc(&g.d_shard_off, (uint64_t)S + 1));
  k_starts<<<grid_for(E + 1), 256, 0, st>>>(K, E, bsrc + bn, ~0ull, S,
                                            (uint32_t*)start.p);
  k_counts<<<grid_for((uint64_t)S + 1), 256, 0, st>>>((uint32_t*)start.p, S, g.d_shard_cnt, (uint64_t*)padded.p);
  CK(cudaGetLastError());
  {
    DevBuf t2, scan;
    size_t b2 = 0;
    CK(dalloc((uint64_t**)&scan.p, (uint64_t)S + 1));
    CK(cub::DeviceScan::ExclusiveSum(nullptr, b2, (uint64_t*)padded.p, (uint64_t*)scan.p, (int64_t)S + 1, st));
    CK(dev_alloc(&t2.p, b2 ? b2 : 1, st));
    CK(cub::DeviceScan::ExclusiveSum(t2.p, b2, (uint64_t*)padded.p, (uint64_t*)scan.p, (int64_t)S + 1, st));
    uint64_t P = 0;
    CK(cudaMemcpyAsync(&P, (uint64_t*)scan.p + S, 8, cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
    if (P >= 0xFFFFFFF0ull) { err = "padded entry count exceeds 32-bit positions"; return CUSHA_EINVAL; }
    g.P = P;
    k_narrow<<<grid_for((uint64_t)S + 1), 256, 0, st>>>((uint64_t*)scan.p, (uint64_t)S + 1, g.d_shard_off);
    CK(cudaGetLastError());
  }
  const uint64_t P = g.P;
  CK(dalloc(&g.d_dest, P));
  CK(dalloc(&g.d_srcloc, P));
  if (g.keep_ids) CK(dalloc(&g.d_eid, P));  // layout inspection only (no kernel reads it)
  if (d_val) { CK(dalloc(&g.d_ev, P)); g.has_ev = true; }
  pt.mark("offsets + alloc shard arrays");
  if (chunks && chunks->n) CK(cudaStreamWaitEvent(st, chunks->all, 0));  // the edge values' copy trails the src/dst chunks
  if (d_val && E) {
    k_max_abs_f32<<<grid_for(E), 256, 0, st>>>(d_val, E, (uint32_t*)mx.p + 1);
    CK(cudaMemcpyAsync(&ev_bits, (uint32_t*)mx.p + 1, 4, cudaMemcpyDeviceToHost, st));
  }
  k_fill_shard_pads<<<grid_for((uint64_t)S * kPad), 256, 0, st>>>(g.d_shard_off, g.d_shard_cnt, S, N, g.d_dest,
                                                                   g.d_srcloc, g.d_eid, g.d_ev);
  if (E)
    k_scatter_gs<<<grid_for(E), 256, 0, st>>>(K, I, E, (uint32_t*)start.p, g.d_shard_off, bn, bsrc, d_val, N, g.d_dest,
                                              g.d_srcloc, g.d_eid, g.d_ev);
  // the in-degree count only reads DestIndex: a side stream runs it beside the
  // window table and CW (joined before the build returns)
  struct Side {
    cudaStream_t s = nullptr;
    cudaEvent_t fork = nullptr, join = nullptr;
    ~Side() {
      if (s) { cudaStreamSynchronize(s); cudaStreamDestroy(s); }
      if (fork) cudaEventDestroy(fork);
      if (join) cudaEventDestroy(join);
    }
  } side;
  CK(cudaStreamCreateWithFlags(&side.s, cudaStreamNonBlocking));
  CK(cudaEventCreateWithFlags(&side.fork, cudaEventDisableTiming));
  CK(cudaEventCreateWithFlags(&side.join, cudaEventDisableTiming));
  CK(cudaEventRecord(side.fork, st));
  CK(cudaStreamWaitEvent(side.s, side.fork, 0));
  if (hist_indeg && E) {
    if (4ull * N > 48 * 1024)
      CK(cudaFuncSetAttribute(k_indeg_max, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)(4 * N)));
    k_indeg_max<<<S, 256, 4 * N, side.s>>>(g.d_dest, g.d_shard_off, g.d_shard_cnt, N, (uint32_t*)mx.p);
  }
  CK(cudaMemcpyAsync(h, mx.p, 4, cudaMemcpyDeviceToHost, side.s));
  CK(cudaEventRecord(side.join, side.s));
  CK(cudaGetLastError());

  // ---- window table W_ij (both representations keep it; GS stage 4 reads it)
  pt.mark("scatter shards");
  CK(dalloc(&g.d_win, ((uint64_t)S + 1) * S));
  if (E)
    k_windows<<<grid_for(E), 256, 0, st>>>(K, E, (uint32_t*)start.p, g.d_shard_off, N, S, bn, bsrc, g.d_win);
  k_windows_tail<<<grid_for(S), 256, 0, st>>>(K, (uint32_t*)start.p, g.d_shard_off, g.d_shard_cnt, N, S, bn, bsrc,
                                              g.d_win);
  CK(cudaGetLastError());

  // ---- out-degrees (PR NbrsNum, L318) and |CW_i|
  pt.mark("window table");
  CK(dalloc(&g.d_cw_cnt, S));
  k_cw_counts<<<S, 256, 0, st>>>(g.d_outdeg, V, N, g.d_cw_cnt);
  CK(cudaGetLastError());

  CK(dalloc(&g.d_active, S));  // stage-4 prefetch predictor of the shard pass
  if (g.skip_clean) CK(dalloc(&g.d_dirty, S));
  CK(dalloc(&g.d_shard_seq, S));  // overlapped passes: per-shard pass order

  // ---- Concatenated Windows + Mapper (§3.2)
  pt.mark("outdeg + cw counts");
  if (g.repr == CUSHA_REPR_CW) {
    // CW_i offsets: |CW_i| = out-degree sum of shard i (cw_cnt), padded to kPad
    DevBuf cpad, cscan, t4;
    CK(dalloc((uint64_t**)&cpad.p, (uint64_t)S + 1));
    CK(dalloc((uint64_t**)&cscan.p, (uint64_t)S + 1));
    k_pad_counts<<<grid_for((uint64_t)S + 1), 256, 0, st>>>(g.d_cw_cnt, S, (uint64_t*)cpad.p);
    CK(cudaGetLastError());
    size_t b4 = 0;
    CK(cub::DeviceScan::ExclusiveSum(nullptr, b4, (uint64_t*)cpad.p, (uint64_t*)cscan.p, (int64_t)S + 1, st));
    CK(dev_alloc(&t4.p, b4 ? b4 : 1, st));
    CK(cub::DeviceScan::ExclusiveSum(t4.p, b4, (uint64_t*)cpad.p, (uint64_t*)cscan.p, (int64_t)S + 1, st));
    uint64_t Q = 0;
    CK(cudaMemcpyAsync(&Q, (uint64_t*)cscan.p + S, 8, cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
    if (Q >= 0xFFFFFFF0ull) { err = "padded CW entry count exceeds 32-bit positions"; return CUSHA_EINVAL; }
    g.Q = Q;
    CK(dalloc(&g.d_cw_off, (uint64_t)S + 1));
    k_narrow<<<grid_for((uint64_t)S + 1), 256, 0, st>>>((uint64_t*)cscan.p, (uint64_t)S + 1, g.d_cw_off);
    CK(dalloc(&g.d_cw_src, Q));
    CK(dalloc(&g.d_mapper, Q));
    CK(dalloc(&g.d_cw_win, Q));
    CK(dalloc(&g.d_cw_delta, (uint64_t)S * S));
    k_fill_cw_pads<<<grid_for((uint64_t)S * kPad), 256, 0, st>>>(g.d_cw_off, g.d_cw_cnt, S, (uint32_t)P,
                                                                  g.d_cw_src, g.d_mapper, g.d_cw_win);
    if (E)
      k_cw_from_windows<<<S, 256, 0, st>>>(g.d_win, S, g.d_cw_off, g.d_srcloc, g.d_cw_src, g.d_mapper, g.d_cw_win,
                                           g.d_cw_delta);
    CK(cudaGetLastError());
    CK(cudaStreamSynchronize(st));
    // CW keeps the 3-tuple shards + SrcIndexCW + Mapper (L175): no per-entry SrcIndex in shard order
    cudaFreeAsync(g.d_srcloc, st);
    g.d_srcloc = nullptr;
    pt.mark("CW offsets + scatter");
    if (kernels_rle()) {  // the run-length Mapper only serves builds with CUSHA_RLE stage 4
      const int rc = build_runs(g, err);
      if (rc) return rc;
    }
  }
  pt.mark("Mapper runs");
  CK(cudaStreamWaitEvent(st, side.join, 0));
  CK(cudaStreamSynchronize(st));
  std::memcpy(&g.max_abs_ev, &ev_bits, 4);
  g.max_indeg = h[0];
  return CUSHA_OK;
}

// ------------------------------------------------ host-streamed topology (row f3)
// "If graphs do not fit in the GPU RAM, a multi-streamed procedure should be
// incorporated to overlap computation and data transfer" (L455).  Shards
// [host_shard, S) keep their per-entry arrays (DestIndex, EdgeValue, SrcIndex,
// edge ids) and, for CW, CW_i's SrcIndexCW and Mapper in pinned, mapped host
// memory; the shard pass's TMA ring streams them over the host link each pass
// exactly as it streams HBM tiles, so the transfer overlaps the consumers'
// work tile by tile.  SrcValue, VertexValues and
// the O(V + S^2) arrays stay in HBM.  host_shard is the first shard whose
// prefix of per-entry arrays would exceed topo_budget bytes of HBM.
namespace {
template <class T>
int move_tail(T*& dev, T*& host, uint64_t n, uint64_t split, cudaStream_t st, uint64_t& host_bytes,
              std::string& err) {
  if (!dev || split >= n) return CUSHA_OK;
  const uint64_t m = n - split;
  void* hp = nullptr;
  CK(cudaHostAlloc(&hp, m * sizeof(T), cudaHostAllocMapped | cudaHostAllocPortable));
  void* dp = nullptr;
  CK(cudaHostGetDevicePointer(&dp, hp, 0));
  if (dp != hp) {  // UVA: the mapped allocation has one address on host and device
    cudaFreeHost(hp);
    err = "mapped host memory without a unified address";
    return CUSHA_EUNSUPPORTED;
  }
  host = static_cast<T*>(hp);
  CK(cudaMemcpyAsync(host, dev + split, m * sizeof(T), cudaMemcpyDeviceToHost, st));
  T* nd = nullptr;
  if (split) {
    CK(dalloc(&nd, split));
    CK(cudaMemcpyAsync(nd, dev, split * sizeof(T), cudaMemcpyDeviceToDevice, st));
  }
  CK(cudaFreeAsync(dev, st));
  dev = nd;
  host_bytes += m * sizeof(T);
  return CUSHA_OK;
}
}  // namespace

int offload_topology(Graph& g, std::string& err) {
  cudaStream_t st = g.stream;
  t_alloc_stream = st;
  const uint32_t S = g.Sl;  // the graph's (partition's) own shards
  g.splitP = g.P;
  g.splitQ = g.Q;
  g.host_shard = S;
  if (!g.topo_budget || !S) return CUSHA_OK;
  std::vector<uint32_t> so(S + 1), co(S + 1, 0);
  CK(cudaMemcpyAsync(so.data(), g.d_shard_off, 4ull * (S + 1), cudaMemcpyDeviceToHost, st));
  if (g.d_cw_off) CK(cudaMemcpyAsync(co.data(), g.d_cw_off, 4ull * (S + 1), cudaMemcpyDeviceToHost, st));
  CK(cudaStreamSynchronize(st));
  const uint64_t bP = 2 + (g.d_eid ? 4 : 0) + (g.has_ev ? 4 : 0) + (g.d_srcloc ? 2 : 0);  // DestIndex, edge id, EdgeValue, SrcIndex
  const uint64_t bQ = g.d_cw_src ? 8 : 0;                                                 // SrcIndexCW, Mapper, window
  uint32_t h = 0;
  while (h < S && (uint64_t)so[h + 1] * bP + (uint64_t)co[h + 1] * bQ <= g.topo_budget) ++h;
  g.host_shard = h;
  g.splitP = so[h];
  g.splitQ = g.d_cw_src ? co[h] : g.Q;
  int rc;
  if ((rc = move_tail(g.d_dest, g.h_dest, g.P, g.splitP, st, g.host_bytes, err)) ||
      (rc = move_tail(g.d_ev, g.h_ev, g.P, g.splitP, st, g.host_bytes, err)) ||
      (rc = move_tail(g.d_eid, g.h_eid, g.P, g.splitP, st, g.host_bytes, err)) ||
      (rc = move_tail(g.d_srcloc, g.h_srcloc, g.P, g.splitP, st, g.host_bytes, err)) ||
      (rc = move_tail(g.d_cw_src, g.h_cw_src, g.Q, g.splitQ, st, g.host_bytes, err)) ||
      (rc = move_tail(g.d_mapper, g.h_mapper, g.Q, g.splitQ, st, g.host_bytes, err)) ||
      (rc = move_tail(g.d_cw_win, g.h_cw_win, g.Q, g.splitQ, st, g.host_bytes, err)))
    return rc;
  CK(cudaStreamSynchronize(st));
  return CUSHA_OK;
}

// ------------------------------------------------ destination-range partition
// Contiguous shard ranges (= destination-vertex ranges, the Partitioned
// property) with near-equal work: bounds[q] = first shard whose work
// prefix reaches q/G of the total.
void partition_bounds(uint32_t S, const uint64_t* work, uint32_t G, uint32_t* bounds) {
  uint64_t total = 0;
  for (uint32_t s = 0; s < S; ++s) total += work[s];
  bounds[0] = 0;
  uint64_t pre = 0;
  uint32_t s = 0;
  for (uint32_t q = 1; q < G; ++q) {
    const long double target = (long double)total * q / G;
    while (s < S && (long double)pre + (long double)work[s] / 2 < target) pre += work[s++];
    bounds[q] = s;
  }
  bounds[G] = S;
}

void free_device_arrays(Graph& g) {
  void* ptrs[] = {g.d_shard_off, g.d_shard_cnt, g.d_dest, g.d_srcloc, g.d_eid, g.d_ev, g.d_win, g.d_cw_off,
                  g.d_cw_cnt, g.d_cw_src, g.d_mapper, g.d_outdeg, g.d_ctl, g.d_trace, g.d_sync_peer,
                  g.d_active, g.d_bounds, g.d_owner, g.d_cwp, g.d_run_k, g.d_run_t, g.d_sv_peer, g.d_dirty_peer,
                  g.d_run_unit, g.d_run_bits, g.d_run_d, g.d_shard_seq, g.d_cw_win, g.d_cw_delta, g.d_order,
                  g.d_init_chunks};
  for (void* p : ptrs)
    if (p) cudaFreeAsync(p, g.stream);
  if (g.d_dirty) {
    if (g.srcvalue_ipc) cudaFree(g.d_dirty);
    else cudaFreeAsync(g.d_dirty, g.stream);
  }
  if (g.d_srcvalue) {
    if (g.srcvalue_ipc) cudaFree(g.d_srcvalue);  // IPC-exported allocations are not stream-ordered
    else cudaFreeAsync(g.d_srcvalue, g.stream);
  }
  if (g.d_srcvalue2) cudaFreeAsync(g.d_srcvalue2, g.stream);
  if (g.d_vv) {
    if (g.srcvalue_ipc) cudaFree(g.d_vv);
    else cudaFreeAsync(g.d_vv, g.stream);
  }
  if (g.d_sync) cudaFree(g.d_sync);
  g.d_sync = nullptr;
  g.d_sync_peer = nullptr;
  g.vv_peer.clear();
  g.connected = false;
  g.d_srcvalue2 = nullptr;
  for (void*& p : g.d_init)
    if (p) { cudaFreeAsync(p, g.stream); p = nullptr; }
  for (void* p : g.ipc_open) cudaIpcCloseMemHandle(p);
  g.ipc_open.clear();
  void* hosts[] = {g.h_dest, g.h_ev, g.h_srcloc, g.h_eid, g.h_cw_src, g.h_mapper, g.h_cw_win};
  for (void* p : hosts)
    if (p) cudaFreeHost(p);
  g.d_shard_off = g.d_shard_cnt = g.d_win = g.d_cw_off = g.d_cw_cnt = g.d_mapper = g.d_outdeg = nullptr;
  g.d_dest = g.d_srcloc = g.d_cw_src = g.d_cw_win = nullptr;
  g.d_eid = g.d_ev = g.d_bounds = g.d_cwp = g.d_run_k = g.d_run_t = g.d_run_unit = g.d_run_bits = g.d_run_d = nullptr;
  g.d_shard_seq = g.d_cw_delta = g.d_dirty = g.d_srcvalue = g.d_order = nullptr;
  g.d_init_chunks = nullptr;
  g.init_nchunks = 0;
  g.d_vv = nullptr; g.d_ctl = nullptr; g.d_trace = nullptr; g.d_active = nullptr; g.d_owner = nullptr;
  g.d_sv_peer = nullptr; g.d_dirty_peer = nullptr;
  g.h_dest = nullptr; g.h_ev = nullptr; g.h_srcloc = nullptr; g.h_eid = nullptr; g.h_cw_src = nullptr;
  g.h_mapper = nullptr; g.h_cw_win = nullptr;
}

// The library's device memory comes from a private stream-ordered pool per
// device whose release threshold keeps freed blocks mapped, so that repeated
// builds (the e2e path) reuse them.  It is private: torch's caching allocator,
// NCCL and other cudaMalloc users of the process keep the default pool's
// behaviour.  cusha_trim_memory() returns the unused blocks to the device.
static cudaError_t pool_of(int dev, cudaMemPool_t* out) {
  static cudaMemPool_t pools[64] = {};
  static bool made[64] = {};
  if (dev < 0 || dev >= 64) return cudaErrorInvalidDevice;
  if (!made[dev]) {
    cudaMemPoolProps props = {};
    props.allocType = cudaMemAllocationTypePinned;
    props.location.type = cudaMemLocationTypeDevice;
    props.location.id = dev;
    const cudaError_t e = cudaMemPoolCreate(&pools[dev], &props);
    if (e != cudaSuccess) return e;
    uint64_t keep = UINT64_MAX;
    cudaMemPoolSetAttribute(pools[dev], cudaMemPoolAttrReleaseThreshold, &keep);
    made[dev] = true;
  }
  *out = pools[dev];
  return cudaSuccess;
}

cudaError_t dev_alloc(void** p, size_t bytes, cudaStream_t s) {
  int dev = 0;
  cudaError_t e = cudaGetDevice(&dev);
  cudaMemPool_t pool;
  if (e == cudaSuccess) e = pool_of(dev, &pool);
  if (e != cudaSuccess) return e;
  return cudaMallocFromPoolAsync(p, bytes ? bytes : 1, pool, s);
}

cudaError_t trim_pool(int dev) {
  cudaMemPool_t pool;
  cudaError_t e = pool_of(dev, &pool);
  if (e == cudaSuccess) e = cudaMemPoolTrimTo(pool, 0);
  return e;
}

}  // namespace cusha
