// partition.cu — row e / row f3: the layout of a destination-range partition
// built straight from the edge list, without building the whole graph first.
//
// Everything a partition needs besides its own edges follows from one table,
// the shard-pair counts C[i][j] = #edges whose source lies in shard i and
// whose destination lies in shard j (|W_ij|, the window sizes of L155):
//  - shard j holds sum_i C[i][j] entries and CW_i holds sum_j C[i][j] (L179),
//    which give the padded offsets of both inside the owning partitions and
//    the per-shard work that places the partition bounds;
//  - W_ij starts inside shard j at sum_{i' < i} C[i'][j] (Ordered, L129: a
//    shard lists its entries by SrcIndex), and inside CW_i at sum_{j' < j}
//    C[i][j'] (CW_i lists W_i0, W_i1, ... in j order, L175), so a CW entry's
//    Mapper target in the owner of j is the window's start in shard j plus
//    the entry's rank inside the window.
// So a partition sorts only its own in-edges (its shards, key (shard(dst),
// src, dst mod N), input order breaking ties - R17, as the single-GPU build)
// and its own out-edges (the CW of its source shards, key (shard(src), j,
// src mod N, dst mod N)), and the result is exactly the global layout's slice
// (tests/test_gpu_partition.py checks that).  The edge list is streamed in
// chunks (from host or device memory), so device memory during the build is
// one chunk plus one partition's sort - not the whole graph: with the
// partitions' topology kept in pinned host memory this is the out-of-core
// path of L455 (row f3), and one process per GPU builds only its own rank.
// Positions are 32-bit and local to a partition.
#include <cub/cub.cuh>

#include <algorithm>
#include <cstring>
#include <string>
#include <vector>

#include "common.cuh"
#include "graph.hpp"

namespace cusha {

namespace {

#define CKP(call)                                                                    \
  do {                                                                               \
    cudaError_t e_ = (call);                                                         \
    if (e_ != cudaSuccess) {                                                         \
      err = std::string(#call) + ": " + cudaGetErrorString(e_);                      \
      return e_ == cudaErrorMemoryAllocation ? CUSHA_ENOMEM : CUSHA_ECUDA;           \
    }                                                                                \
  } while (0)

#define GSTRIDE(i, n) for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < (n); i += (uint64_t)gridDim.x * blockDim.x)

inline unsigned grid_of(uint64_t n, unsigned block = 256) {
  uint64_t g = (n + block - 1) / block;
  if (g > 148ull * 64) g = 148ull * 64;
  return (unsigned)(g ? g : 1);
}

int nbits(uint64_t maxval) {
  int b = 0;
  while (b < 64 && (1ull << b) <= maxval) ++b;
  return b ? b : 1;
}

struct Buf {  // stream-ordered temporary
  void* p = nullptr;
  cudaStream_t s = nullptr;
  ~Buf() { if (p) cudaFreeAsync(p, s); }
};
template <class T>
cudaError_t alloc(Buf& b, uint64_t n, cudaStream_t s) {
  b.s = s;
  return dev_alloc(&b.p, (n ? n : 1) * sizeof(T), s);
}
template <class T>
T* ptr(const Buf& b) { return static_cast<T*>(b.p); }

// ---------------------------------------------------------------- chunks
// The edge list in chunks of at most kChunk edges, as device pointers: a
// slice of device-resident inputs, or a staged copy of host inputs (two
// staging buffers; the copy of chunk c+1 overlaps the kernels of chunk c).
constexpr uint64_t kChunkEdges = 1ull << 27;
struct ChunkSource {
  const uint32_t *src, *dst, *val;
  uint64_t E;
  bool host;
  cudaStream_t st, cs = nullptr;
  Buf stage[2];
  cudaEvent_t copied[2] = {}, used[2] = {};
  int init(std::string& err) {
    if (!host) return CUSHA_OK;
    const uint64_t n = std::min(E, kChunkEdges), w = val ? 3 : 2;
    for (int b = 0; b < 2; ++b) {
      CKP(alloc<uint32_t>(stage[b], n * w, st));
      CKP(cudaEventCreateWithFlags(&copied[b], cudaEventDisableTiming));
      CKP(cudaEventCreateWithFlags(&used[b], cudaEventDisableTiming));
      CKP(cudaEventRecord(used[b], st));  // the staging allocation precedes the first copy
    }
    CKP(cudaStreamCreateWithFlags(&cs, cudaStreamNonBlocking));
    return CUSHA_OK;
  }
  ~ChunkSource() {
    if (cs) { cudaStreamSynchronize(cs); cudaStreamDestroy(cs); }
    for (int b = 0; b < 2; ++b) {
      if (copied[b]) cudaEventDestroy(copied[b]);
      if (used[b]) cudaEventDestroy(used[b]);
    }
  }
  uint64_t count() const { return (E + kChunkEdges - 1) / kChunkEdges; }
  // chunk c's device pointers, valid on st until release(c); chunks are
  // requested in order, and the copy of chunk c + 1 is issued with chunk c
  uint64_t issued = 0;
  int get(uint64_t c, const uint32_t** s, const uint32_t** d, const uint32_t** v, uint64_t* lo, uint64_t* n,
          std::string& err) {
    *lo = c * kChunkEdges;
    *n = std::min(kChunkEdges, E - *lo);
    if (!host) {
      *s = src + *lo; *d = dst + *lo; *v = val ? val + *lo : nullptr;
      return CUSHA_OK;
    }
    const uint64_t cap = std::min(E, kChunkEdges);
    for (; issued < std::min(c + 2, count()); ++issued) {
      const uint64_t k = issued;
      const int b = (int)(k & 1);
      const uint64_t l = k * kChunkEdges, m = std::min(kChunkEdges, E - l);
      uint32_t* t = ptr<uint32_t>(stage[b]);
      CKP(cudaStreamWaitEvent(cs, used[b], 0));  // chunk k - 2 released the buffer
      CKP(cudaMemcpyAsync(t, src + l, m * 4, cudaMemcpyHostToDevice, cs));
      CKP(cudaMemcpyAsync(t + cap, dst + l, m * 4, cudaMemcpyHostToDevice, cs));
      if (val) CKP(cudaMemcpyAsync(t + 2 * cap, val + l, m * 4, cudaMemcpyHostToDevice, cs));
      CKP(cudaEventRecord(copied[b], cs));
    }
    const int b = (int)(c & 1);
    CKP(cudaStreamWaitEvent(st, copied[b], 0));
    uint32_t* t = ptr<uint32_t>(stage[b]);
    *s = t; *d = t + cap; *v = val ? t + 2 * cap : nullptr;
    return CUSHA_OK;
  }
  int release(uint64_t c, std::string& err) {
    if (host) CKP(cudaEventRecord(used[c & 1], st));
    return CUSHA_OK;
  }
};

// ----------------------------------------------------------------- plan
__global__ void k_pair_hist(const uint32_t* __restrict__ src, const uint32_t* __restrict__ dst, uint64_t n, uint32_t V,
                            uint32_t N, uint32_t S, uint32_t* C, uint32_t* outdeg, uint32_t* indeg, uint32_t* bad) {
  GSTRIDE(e, n) {
    const uint32_t s = src[e], d = dst[e];
    if (s >= V || d >= V) { *bad = 1; continue; }
    atomicAdd(&C[(uint64_t)(s / N) * S + d / N], 1u);
    atomicAdd(&outdeg[s], 1u);
    atomicAdd(&indeg[d], 1u);
  }
}
__global__ void k_max_u32p(const uint32_t* __restrict__ a, uint64_t n, uint32_t* out) {
  uint32_t m = 0;
  GSTRIDE(i, n) m = max(m, a[i]);
  for (int o = 16; o; o >>= 1) m = max(m, __shfl_xor_sync(0xFFFFFFFFu, m, o));
  if ((threadIdx.x & 31) == 0 && m) atomicMax(out, m);
}
__global__ void k_max_abs_bits(const uint32_t* __restrict__ a, uint64_t n, uint32_t* out) {
  uint32_t m = 0;
  GSTRIDE(i, n) {
    uint32_t b = a[i] & 0x7FFFFFFFu;
    if (b > 0x7F800000u) b = 0x7F800000u;
    m = max(m, b);
  }
  for (int o = 16; o; o >>= 1) m = max(m, __shfl_xor_sync(0xFFFFFFFFu, m, o));
  if ((threadIdx.x & 31) == 0 && m) atomicMax(out, m);
}
// column j: win[i][j] = offl[j] + sum_{i' < i} C[i'][j] for i = 0..S (the window table, positions local to owner(j))
__global__ void k_win_from_counts(const uint32_t* __restrict__ C, const uint32_t* __restrict__ offl, uint32_t S,
                                  uint32_t* win) {
  GSTRIDE(j, (uint64_t)S) {
    uint32_t acc = offl[j];
    for (uint32_t i = 0; i < S; ++i) {
      win[(uint64_t)i * S + j] = acc;
      acc += C[(uint64_t)i * S + j];
    }
    win[(uint64_t)S * S + j] = acc;
  }
}
// row i: R[i][j] = sum_{j' < j} C[i][j'] (where W_ij starts inside CW_i)
__global__ void k_row_prefix(const uint32_t* __restrict__ C, uint32_t S, uint32_t* R) {
  GSTRIDE(i, (uint64_t)S) {
    uint32_t acc = 0;
    for (uint32_t j = 0; j < S; ++j) {
      R[i * (uint64_t)S + j] = acc;
      acc += C[i * (uint64_t)S + j];
    }
  }
}

// ------------------------------------------------------------ partition
struct InRange {
  const uint32_t* a;
  uint32_t lo, hi;
  __device__ bool operator()(uint64_t e) const { const uint32_t x = a[e]; return x >= lo && x < hi; }
};
// keys of the selected in-edges: (shard(dst) - s0 | src | dst mod N); payload = selection index (input order)
__global__ void k_in_keys(const uint32_t* __restrict__ src, const uint32_t* __restrict__ dst,
                          const uint32_t* __restrict__ val, const uint64_t* __restrict__ sel, uint64_t n, uint64_t base,
                          uint32_t N, uint32_t s0, int bn, int bsrc, uint64_t* keys, uint32_t* ids, uint32_t* vsel,
                          uint32_t* gid) {
  GSTRIDE(t, n) {
    const uint64_t e = sel[t];
    const uint32_t s = src[e], d = dst[e];
    keys[t] = ((uint64_t)(d / N - s0) << (bsrc + bn)) | ((uint64_t)s << bn) | (uint64_t)(d % N);
    ids[t] = (uint32_t)(base + t);
    if (vsel) vsel[base + t] = val[e];
    if (gid) gid[base + t] = (uint32_t)e;  // chunk-relative; the caller adds the chunk base
  }
}
__global__ void k_add(uint32_t* a, uint64_t n, uint32_t x) { GSTRIDE(i, n) a[i] += x; }
// keys of the selected out-edges: (shard(src) - s0 | j | src mod N | dst mod N)
__global__ void k_out_keys(const uint32_t* __restrict__ src, const uint32_t* __restrict__ dst,
                           const uint64_t* __restrict__ sel, uint64_t n, uint32_t N, uint32_t s0, int bn, int bj,
                           uint64_t* keys) {
  GSTRIDE(t, n) {
    const uint64_t e = sel[t];
    const uint32_t s = src[e], d = dst[e];
    keys[t] = ((uint64_t)(s / N - s0) << (bj + 2 * bn)) | ((uint64_t)(d / N) << (2 * bn)) |
              ((uint64_t)(s % N) << bn) | (uint64_t)(d % N);
  }
}
// sorted in-edge p -> padded shard position: local shard sl = key >> (bsrc + bn)
__global__ void k_in_scatter(const uint64_t* __restrict__ keys, const uint32_t* __restrict__ ids, uint64_t n,
                             const uint32_t* __restrict__ start, const uint32_t* __restrict__ off, int bn, int bsrc,
                             const uint32_t* __restrict__ vsel, const uint32_t* __restrict__ gid, uint16_t* dest,
                             uint32_t* ev, uint32_t* eid) {
  const uint64_t mn = (1ull << bn) - 1;
  GSTRIDE(p, n) {
    const uint64_t k = keys[p];
    const uint32_t sl = (uint32_t)(k >> (bsrc + bn));
    const uint32_t pos = off[sl] + (uint32_t)(p - start[sl]);
    dest[pos] = (uint16_t)(k & mn);
    if (ev) ev[pos] = vsel[ids[p]];
    if (eid) eid[pos] = gid[ids[p]];
  }
}
__global__ void k_in_pads(const uint32_t* off, const uint32_t* cnt, uint32_t Sl, uint32_t N, uint16_t* dest,
                          uint32_t* ev, uint32_t* eid) {
  GSTRIDE(i, (uint64_t)Sl * kPad) {
    const uint32_t s = (uint32_t)(i / kPad), r = (uint32_t)(i % kPad);
    const uint32_t pos = off[s] + cnt[s] + r;
    if (pos < off[s + 1]) {
      dest[pos] = (uint16_t)N;
      if (ev) ev[pos] = 0;
      if (eid) eid[pos] = 0xFFFFFFFFu;
    }
  }
}
// sorted out-edge p -> CW position k of CW_i; Mapper = window start in shard j (owner-local) + rank in window
__global__ void k_cw_scatter(const uint64_t* __restrict__ keys, uint64_t n, const uint32_t* __restrict__ cstart,
                             const uint32_t* __restrict__ coff, const uint32_t* __restrict__ win,
                             const uint32_t* __restrict__ R, uint32_t S, uint32_t s0, int bn, int bj, uint16_t* cw_src,
                             uint16_t* cw_win, uint32_t* mapper) {
  const uint64_t mn = (1ull << bn) - 1, mj = (1ull << bj) - 1;
  GSTRIDE(p, n) {
    const uint64_t k = keys[p];
    const uint32_t il = (uint32_t)(k >> (bj + 2 * bn));
    const uint32_t j = (uint32_t)((k >> (2 * bn)) & mj);
    const uint32_t i = s0 + il;
    const uint32_t pos = coff[il] + (uint32_t)(p - cstart[il]);
    const uint32_t ws = coff[il] + R[(uint64_t)i * S + j];  // W_ij's first CW position
    cw_src[pos] = (uint16_t)((k >> bn) & mn);
    cw_win[pos] = (uint16_t)j;
    mapper[pos] = win[(uint64_t)i * S + j] + (pos - ws);
  }
}
__global__ void k_cw_pads(const uint32_t* coff, const uint32_t* ccnt, uint32_t Sl, uint16_t* cw_src, uint16_t* cw_win,
                          uint32_t* mapper) {
  GSTRIDE(i, (uint64_t)Sl * kPad) {
    const uint32_t s = (uint32_t)(i / kPad), r = (uint32_t)(i % kPad);
    const uint32_t pos = coff[s] + ccnt[s] + r;
    if (pos < coff[s + 1]) {
      cw_src[pos] = 0;
      cw_win[pos] = 0xFFFFu;
      mapper[pos] = 0xFFFFFFFFu;
    }
  }
}
// delta[il][j] = (window start in shard j) - (window start in CW_i)  (mod 2^32)
__global__ void k_delta(const uint32_t* __restrict__ win, const uint32_t* __restrict__ R,
                        const uint32_t* __restrict__ coff, uint32_t S, uint32_t s0, uint32_t Sl, uint32_t* delta) {
  GSTRIDE(t, (uint64_t)Sl * S) {
    const uint32_t il = (uint32_t)(t / S), j = (uint32_t)(t % S), i = s0 + il;
    delta[t] = win[(uint64_t)i * S + j] - (coff[il] + R[(uint64_t)i * S + j]);
  }
}
// cwp[il][q] = first CW_i position aimed at partition q; cwp[il][G] = end of CW_i
__global__ void k_cwp(const uint32_t* __restrict__ R, const uint32_t* __restrict__ coff,
                      const uint32_t* __restrict__ ccnt, const uint32_t* __restrict__ bounds, uint32_t S, uint32_t s0,
                      uint32_t Sl, uint32_t G, uint32_t* cwp) {
  GSTRIDE(t, (uint64_t)Sl * (G + 1)) {
    const uint32_t il = (uint32_t)(t / (G + 1)), q = (uint32_t)(t % (G + 1)), i = s0 + il;
    cwp[t] = coff[il] + (q == G ? ccnt[il] : (bounds[q] < S ? R[(uint64_t)i * S + bounds[q]] : ccnt[il]));
  }
}

uint32_t pad8(uint64_t c) { return (uint32_t)((c + kPad - 1) / kPad * kPad); }

}  // namespace

// --------------------------------------------------------------------------
// Shard-pair counts, degrees and the tables every partition derives from them.
int plan_partitions(const PlanInput& in, uint32_t G, Plan& pl, std::string& err) {
  cudaStream_t st = in.stream;
  const uint32_t V = in.V, N = in.N, S = (V + N - 1) / N;
  pl.V = V; pl.N = N; pl.S = S; pl.E = in.E;
  const uint64_t S2 = (uint64_t)S * S;
  CKP(dev_alloc((void**)&pl.d_C, 4 * std::max<uint64_t>(S2, 1), st));
  CKP(dev_alloc((void**)&pl.d_outdeg, 4ull * V, st));
  Buf indeg, mx;
  CKP(alloc<uint32_t>(indeg, V, st));
  CKP(alloc<uint32_t>(mx, 4, st));
  CKP(cudaMemsetAsync(pl.d_C, 0, 4 * S2, st));
  CKP(cudaMemsetAsync(pl.d_outdeg, 0, 4ull * V, st));
  CKP(cudaMemsetAsync(indeg.p, 0, 4ull * V, st));
  CKP(cudaMemsetAsync(mx.p, 0, 16, st));
  ChunkSource cs{in.src, in.dst, in.val, in.E, in.host, st};
  int rc = cs.init(err);
  if (rc) return rc;
  for (uint64_t c = 0; c < cs.count(); ++c) {
    const uint32_t *s, *d, *v;
    uint64_t lo, n;
    if ((rc = cs.get(c, &s, &d, &v, &lo, &n, err))) return rc;
    k_pair_hist<<<grid_of(n), 256, 0, st>>>(s, d, n, V, N, S, pl.d_C, pl.d_outdeg, ptr<uint32_t>(indeg),
                                            ptr<uint32_t>(mx) + 2);
    if (v) k_max_abs_bits<<<grid_of(n), 256, 0, st>>>(v, n, ptr<uint32_t>(mx) + 1);
    if ((rc = cs.release(c, err))) return rc;
  }
  k_max_u32p<<<grid_of(V), 256, 0, st>>>(ptr<uint32_t>(indeg), V, ptr<uint32_t>(mx));
  CKP(cudaGetLastError());
  uint32_t h[3];
  CKP(cudaMemcpyAsync(h, mx.p, 12, cudaMemcpyDeviceToHost, st));
  std::vector<uint32_t> C(S2);
  CKP(cudaMemcpyAsync(C.data(), pl.d_C, 4 * S2, cudaMemcpyDeviceToHost, st));
  CKP(cudaStreamSynchronize(st));
  if (h[2]) { err = "edge endpoint >= num_vertices"; return CUSHA_EINVAL; }
  pl.max_indeg = h[0];
  std::memcpy(&pl.max_abs_ev, &h[1], 4);
  // shard sizes (column sums) and CW sizes (row sums), host
  pl.in.assign(S, 0);
  pl.out.assign(S, 0);
  for (uint32_t i = 0; i < S; ++i)
    for (uint32_t j = 0; j < S; ++j) {
      const uint32_t c = C[(uint64_t)i * S + j];
      pl.out[i] += c;
      pl.in[j] += c;
    }
  std::vector<uint64_t> work(S);
  for (uint32_t s = 0; s < S; ++s) work[s] = (uint64_t)pl.in[s] + pl.out[s];
  const uint32_t Gp = std::max<uint32_t>(1, std::min<uint32_t>(G, S));
  pl.bounds.assign(Gp + 1, 0);
  partition_bounds(S, work.data(), Gp, pl.bounds.data());
  // padded offsets of every shard / CW_i inside its owner partition (32-bit, local)
  std::vector<uint32_t> offl(S + 1), coffl(S + 1);
  pl.owner.assign(S, 0);
  for (uint32_t q = 0; q < Gp; ++q) {
    uint64_t a = 0, b = 0;
    for (uint32_t s = pl.bounds[q]; s < pl.bounds[q + 1]; ++s) {
      pl.owner[s] = (uint8_t)q;
      offl[s] = (uint32_t)a;
      coffl[s] = (uint32_t)b;
      a += pad8(pl.in[s]);
      b += pad8(pl.out[s]);
      if (a >= 0xFFFFFFF0ull || b >= 0xFFFFFFF0ull) {
        err = "a partition exceeds 32-bit positions: use more partitions";
        return CUSHA_EINVAL;
      }
    }
  }
  offl[S] = 0;
  coffl[S] = 0;
  pl.offl = offl;
  pl.coffl = coffl;
  Buf doffl;
  CKP(alloc<uint32_t>(doffl, S + 1, st));
  CKP(cudaMemcpyAsync(doffl.p, offl.data(), 4ull * (S + 1), cudaMemcpyHostToDevice, st));
  CKP(dev_alloc((void**)&pl.d_win, 4ull * (S + 1) * S, st));
  CKP(dev_alloc((void**)&pl.d_R, 4 * std::max<uint64_t>(S2, 1), st));
  k_win_from_counts<<<grid_of(S, 128), 128, 0, st>>>(pl.d_C, ptr<uint32_t>(doffl), S, pl.d_win);
  k_row_prefix<<<grid_of(S, 128), 128, 0, st>>>(pl.d_C, S, pl.d_R);
  CKP(cudaGetLastError());
  CKP(cudaStreamSynchronize(st));
  return CUSHA_OK;
}

void free_plan(Plan& pl, cudaStream_t st) {
  void* p[] = {pl.d_C, pl.d_outdeg, pl.d_win, pl.d_R};
  for (void* x : p)
    if (x) cudaFreeAsync(x, st);
  pl.d_C = pl.d_outdeg = pl.d_win = pl.d_R = nullptr;
}

// Stable selection of the edges whose `key` endpoint lies in [lo, hi), chunk
// by chunk; fills the partition's sort input through `emit`.
template <class Emit>
static int select_edges(const PlanInput& in, bool by_src, uint32_t lo, uint32_t hi, Emit&& emit, std::string& err) {
  cudaStream_t st = in.stream;
  ChunkSource cs{in.src, in.dst, in.val, in.E, in.host, st};
  int rc = cs.init(err);
  if (rc) return rc;
  const uint64_t cap = std::min(in.E, kChunkEdges);
  Buf sel, nsel, tmp;
  CKP(alloc<uint64_t>(sel, cap, st));
  CKP(alloc<uint64_t>(nsel, 1, st));
  size_t tb = 0;
  cub::CountingInputIterator<uint64_t> it(0);
  CKP(cub::DeviceSelect::If(nullptr, tb, it, ptr<uint64_t>(sel), ptr<uint64_t>(nsel), (int64_t)cap,
                            InRange{nullptr, lo, hi}, st));
  CKP(alloc<uint8_t>(tmp, tb, st));
  uint64_t base = 0;
  for (uint64_t c = 0; c < cs.count(); ++c) {
    const uint32_t *s, *d, *v;
    uint64_t lo_e, n;
    if ((rc = cs.get(c, &s, &d, &v, &lo_e, &n, err))) return rc;
    size_t tb2 = tb;
    CKP(cub::DeviceSelect::If(tmp.p, tb2, it, ptr<uint64_t>(sel), ptr<uint64_t>(nsel), (int64_t)n,
                              InRange{by_src ? s : d, lo, hi}, st));
    uint64_t m = 0;
    CKP(cudaMemcpyAsync(&m, nsel.p, 8, cudaMemcpyDeviceToHost, st));
    CKP(cudaStreamSynchronize(st));
    if (m && (rc = emit(s, d, v, ptr<uint64_t>(sel), m, base, lo_e, err))) return rc;
    base += m;
    if ((rc = cs.release(c, err))) return rc;
  }
  CKP(cudaStreamSynchronize(st));
  return CUSHA_OK;
}

int build_part_direct(const PlanInput& in, const Plan& pl, uint32_t r, Graph& g, std::string& err) {
  cudaStream_t st = g.stream;
  const uint32_t S = pl.S, N = pl.N, V = pl.V, G = (uint32_t)pl.bounds.size() - 1;
  const uint32_t s0 = pl.bounds[r], s1 = pl.bounds[r + 1], Sl = s1 - s0;
  g.V = V; g.N = N; g.S = S; g.E = pl.E; g.repr = CUSHA_REPR_CW; g.has_ev = in.val != nullptr;
  g.max_indeg = pl.max_indeg; g.max_abs_ev = pl.max_abs_ev;
  g.G = G; g.part = r; g.h_bounds = pl.bounds;
  g.s0 = s0; g.Sl = Sl; g.v0 = s0 * N; g.nvl = (uint32_t)(std::min<uint64_t>(V, (uint64_t)s1 * N) - g.v0);
  // sizes of the partition (host)
  std::vector<uint32_t> off(Sl + 1), coff(Sl + 1), start(Sl + 1), cstart(Sl + 1), cnt(Sl), ccnt(Sl);
  uint64_t P = 0, Q = 0, Ein = 0, Eout = 0;
  for (uint32_t il = 0; il < Sl; ++il) {
    const uint32_t s = s0 + il;
    off[il] = (uint32_t)P; coff[il] = (uint32_t)Q; start[il] = (uint32_t)Ein; cstart[il] = (uint32_t)Eout;
    cnt[il] = pl.in[s]; ccnt[il] = pl.out[s];
    P += pad8(pl.in[s]); Q += pad8(pl.out[s]); Ein += pl.in[s]; Eout += pl.out[s];
  }
  off[Sl] = (uint32_t)P; coff[Sl] = (uint32_t)Q; start[Sl] = (uint32_t)Ein; cstart[Sl] = (uint32_t)Eout;
  g.P = P; g.Q = Q; g.E_loc = Ein;
  const int bn = nbits(N - 1), bsrc = nbits(V - 1), bsl = nbits(Sl ? Sl - 1 : 0), bj = nbits(S - 1);
  if (bsl + bsrc + bn > 64 || bsl + bj + 2 * bn > 64) { err = "partition sort key does not fit 64 bits"; return CUSHA_EINVAL; }
  // small tables
  std::vector<uint8_t> owner(pl.owner);
  CKP(dev_alloc((void**)&g.d_bounds, 4ull * (G + 1), st));
  CKP(dev_alloc((void**)&g.d_owner, std::max<uint32_t>(S, 1), st));
  CKP(dev_alloc((void**)&g.d_shard_off, 4ull * (Sl + 1), st));
  CKP(dev_alloc((void**)&g.d_shard_cnt, 4ull * std::max<uint32_t>(Sl, 1), st));
  CKP(dev_alloc((void**)&g.d_cw_off, 4ull * (Sl + 1), st));
  CKP(dev_alloc((void**)&g.d_cw_cnt, 4ull * std::max<uint32_t>(Sl, 1), st));
  Buf dstart, dcstart;
  CKP(alloc<uint32_t>(dstart, Sl + 1, st));
  CKP(alloc<uint32_t>(dcstart, Sl + 1, st));
  CKP(cudaMemcpyAsync(g.d_bounds, pl.bounds.data(), 4ull * (G + 1), cudaMemcpyHostToDevice, st));
  CKP(cudaMemcpyAsync(g.d_owner, owner.data(), S, cudaMemcpyHostToDevice, st));
  CKP(cudaMemcpyAsync(g.d_shard_off, off.data(), 4ull * (Sl + 1), cudaMemcpyHostToDevice, st));
  CKP(cudaMemcpyAsync(g.d_shard_cnt, cnt.data(), 4ull * Sl, cudaMemcpyHostToDevice, st));
  CKP(cudaMemcpyAsync(g.d_cw_off, coff.data(), 4ull * (Sl + 1), cudaMemcpyHostToDevice, st));
  CKP(cudaMemcpyAsync(g.d_cw_cnt, ccnt.data(), 4ull * Sl, cudaMemcpyHostToDevice, st));
  CKP(cudaMemcpyAsync(dstart.p, start.data(), 4ull * (Sl + 1), cudaMemcpyHostToDevice, st));
  CKP(cudaMemcpyAsync(dcstart.p, cstart.data(), 4ull * (Sl + 1), cudaMemcpyHostToDevice, st));
  const uint32_t v0 = g.v0, v1 = g.v0 + g.nvl;
  int rc;
  // ---- the partition's shards: its in-edges in G-Shards order
  {
    Buf keys, keys2, ids, ids2, vsel, gid, tmp;
    CKP(alloc<uint64_t>(keys, Ein, st));
    CKP(alloc<uint64_t>(keys2, Ein, st));
    CKP(alloc<uint32_t>(ids, Ein, st));
    CKP(alloc<uint32_t>(ids2, Ein, st));
    if (in.val) CKP(alloc<uint32_t>(vsel, Ein, st));
    if (g.keep_ids) CKP(alloc<uint32_t>(gid, Ein, st));
    rc = select_edges(in, false, v0, v1,
                      [&](const uint32_t* s, const uint32_t* d, const uint32_t* v, const uint64_t* sel, uint64_t m,
                          uint64_t base, uint64_t lo_e, std::string& e2) -> int {
                        k_in_keys<<<grid_of(m), 256, 0, st>>>(s, d, v, sel, m, base, N, s0, bn, bsrc,
                                                              ptr<uint64_t>(keys) + base, ptr<uint32_t>(ids) + base,
                                                              in.val ? ptr<uint32_t>(vsel) : nullptr,
                                                              g.keep_ids ? ptr<uint32_t>(gid) : nullptr);
                        if (g.keep_ids) k_add<<<grid_of(m), 256, 0, st>>>(ptr<uint32_t>(gid) + base, m, (uint32_t)lo_e);
                        const cudaError_t ce = cudaGetLastError();
                        if (ce != cudaSuccess) { e2 = cudaGetErrorString(ce); return CUSHA_ECUDA; }
                        return CUSHA_OK;
                      },
                      err);
    if (rc) return rc;
    cub::DoubleBuffer<uint64_t> kb(ptr<uint64_t>(keys), ptr<uint64_t>(keys2));
    cub::DoubleBuffer<uint32_t> vb(ptr<uint32_t>(ids), ptr<uint32_t>(ids2));
    size_t tb = 0;
    if (Ein) {
      CKP(cub::DeviceRadixSort::SortPairs(nullptr, tb, kb, vb, (int64_t)Ein, 0, bsl + bsrc + bn, st));
      CKP(alloc<uint8_t>(tmp, tb, st));
      CKP(cub::DeviceRadixSort::SortPairs(tmp.p, tb, kb, vb, (int64_t)Ein, 0, bsl + bsrc + bn, st));
    }
    CKP(dev_alloc((void**)&g.d_dest, 2 * std::max<uint64_t>(P, 1), st));
    if (in.val) CKP(dev_alloc((void**)&g.d_ev, 4 * std::max<uint64_t>(P, 1), st));
    if (g.keep_ids) CKP(dev_alloc((void**)&g.d_eid, 4 * std::max<uint64_t>(P, 1), st));
    k_in_pads<<<grid_of((uint64_t)Sl * kPad), 256, 0, st>>>(g.d_shard_off, g.d_shard_cnt, Sl, N, g.d_dest, g.d_ev,
                                                             g.d_eid);
    if (Ein)
      k_in_scatter<<<grid_of(Ein), 256, 0, st>>>(kb.Current(), vb.Current(), Ein, ptr<uint32_t>(dstart), g.d_shard_off,
                                                 bn, bsrc, in.val ? ptr<uint32_t>(vsel) : nullptr,
                                                 g.keep_ids ? ptr<uint32_t>(gid) : nullptr, g.d_dest, g.d_ev, g.d_eid);
    CKP(cudaGetLastError());
  }
  // ---- the CW of its source shards: its out-edges in (shard(src), j, src, dst) order
  {
    Buf keys, keys2, tmp;
    CKP(alloc<uint64_t>(keys, Eout, st));
    CKP(alloc<uint64_t>(keys2, Eout, st));
    rc = select_edges(in, true, v0, v1,
                      [&](const uint32_t* s, const uint32_t* d, const uint32_t*, const uint64_t* sel, uint64_t m,
                          uint64_t base, uint64_t, std::string& e2) -> int {
                        k_out_keys<<<grid_of(m), 256, 0, st>>>(s, d, sel, m, N, s0, bn, bj, ptr<uint64_t>(keys) + base);
                        const cudaError_t ce = cudaGetLastError();
                        if (ce != cudaSuccess) { e2 = cudaGetErrorString(ce); return CUSHA_ECUDA; }
                        return CUSHA_OK;
                      },
                      err);
    if (rc) return rc;
    cub::DoubleBuffer<uint64_t> kb(ptr<uint64_t>(keys), ptr<uint64_t>(keys2));
    size_t tb = 0;
    if (Eout) {
      CKP(cub::DeviceRadixSort::SortKeys(nullptr, tb, kb, (int64_t)Eout, 0, bsl + bj + 2 * bn, st));
      CKP(alloc<uint8_t>(tmp, tb, st));
      CKP(cub::DeviceRadixSort::SortKeys(tmp.p, tb, kb, (int64_t)Eout, 0, bsl + bj + 2 * bn, st));
    }
    CKP(dev_alloc((void**)&g.d_cw_src, 2 * std::max<uint64_t>(Q, 1), st));
    CKP(dev_alloc((void**)&g.d_cw_win, 2 * std::max<uint64_t>(Q, 1), st));
    CKP(dev_alloc((void**)&g.d_mapper, 4 * std::max<uint64_t>(Q, 1), st));
    k_cw_pads<<<grid_of((uint64_t)Sl * kPad), 256, 0, st>>>(g.d_cw_off, g.d_cw_cnt, Sl, g.d_cw_src, g.d_cw_win,
                                                            g.d_mapper);
    if (Eout)
      k_cw_scatter<<<grid_of(Eout), 256, 0, st>>>(kb.Current(), Eout, ptr<uint32_t>(dcstart), g.d_cw_off, pl.d_win,
                                                  pl.d_R, S, s0, bn, bj, g.d_cw_src, g.d_cw_win, g.d_mapper);
    CKP(cudaGetLastError());
  }
  // ---- per-source-shard tables: Mapper deltas, segments per target partition, window rows
  CKP(dev_alloc((void**)&g.d_cw_delta, 4 * std::max<uint64_t>((uint64_t)Sl * S, 1), st));
  k_delta<<<grid_of((uint64_t)Sl * S), 256, 0, st>>>(pl.d_win, pl.d_R, g.d_cw_off, S, s0, Sl, g.d_cw_delta);
  CKP(dev_alloc((void**)&g.d_cwp, 4ull * Sl * (G + 1) + 4, st));
  k_cwp<<<grid_of((uint64_t)Sl * (G + 1)), 256, 0, st>>>(pl.d_R, g.d_cw_off, g.d_cw_cnt, g.d_bounds, S, s0, Sl, G,
                                                          g.d_cwp);
  CKP(dev_alloc((void**)&g.d_win, 4ull * (Sl + 1) * S, st));
  CKP(cudaMemcpyAsync(g.d_win, pl.d_win + (uint64_t)s0 * S, 4ull * (Sl + 1) * S, cudaMemcpyDeviceToDevice, st));
  CKP(dev_alloc((void**)&g.d_outdeg, 4ull * std::max<uint32_t>(g.nvl, 1), st));
  CKP(cudaMemcpyAsync(g.d_outdeg, pl.d_outdeg + g.v0, 4ull * g.nvl, cudaMemcpyDeviceToDevice, st));
  CKP(dev_alloc((void**)&g.d_active, std::max<uint32_t>(Sl, 1), st));
  if (g.skip_clean) CKP(dev_alloc((void**)&g.d_dirty, 4ull * std::max<uint32_t>(Sl, 1), st));
  CKP(dev_alloc((void**)&g.d_shard_seq, 4ull * std::max<uint32_t>(Sl, 1), st));
  CKP(cudaGetLastError());
  CKP(cudaStreamSynchronize(st));
  g.splitP = g.P;
  g.splitQ = g.Q;
  g.host_shard = Sl;
  return CUSHA_OK;
}

}  // namespace cusha
