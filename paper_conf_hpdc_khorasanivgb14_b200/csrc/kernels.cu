// kernels.cu — the shard pass (rows a1-a5) and its initialisation kernels.
//
// One launch = one CuSha iteration (Fig. 5): every shard runs the
// four stages once (L191), then the global convergence flag decides whether
// another iteration follows (L189, L255).  The iteration loop stays on the
// device: the last CTA to finish closes the iteration and sets the CUDA-graph
// while-condition, instead of the paper's
// per-iteration cudaMemcpy of is_converged (L189).
//
// Arrays of the partition (a single GPU is one partition, s0 = 0, Sl = S) are
// indexed by the local shard index sl; shard s0 + sl owns global vertices
// [(s0 + sl)*N, ...), held locally at sl*N.
//
// B200 structure: a persistent grid (a few CTAs per
// SM).  In each CTA one producer thread takes shards from a global queue in
// shard order and streams, with the TMA engine (cp.async.bulk), every tile
// the CTA will consume — the shard's entries for stage 2 and, for CW, the
// CW_s index arrays for stage 4 — through a ring of shared-memory slots
// guarded by mbarriers, running ahead across stage and shard boundaries.
// Eight consumer warps run the paper's stages on one shard at a time
// (local_vertices in shared memory, as in Fig. 5), taking tiles from the
// ring.  Stage-4 tiles are prefetched when the shard was active in the
// previous pass (a misprediction only costs bandwidth: an unpredicted active
// shard reads its index arrays directly, a predicted inactive one drops them).
#include <cstdio>
#include <type_traits>
#include <map>
#include <mutex>

#include "algorithms.cuh"
#include "graph.hpp"

namespace cusha {

constexpr uint32_t kFull = 0xFFFFFFFFu;
// tuning constants (tools/tune: variants are built with -DCUSHA_*)
// (measured on C2 PageRank: bytes in flight per SM
// decide; 2 CTAs/SM x 3 slots x 24 KB beat deeper rings at 1 CTA/SM)
#ifndef CUSHA_CONSUMER_WARPS
#define CUSHA_CONSUMER_WARPS 16
#endif
#ifndef CUSHA_STAGES
#define CUSHA_STAGES 3
#endif
#ifndef CUSHA_TILE
#define CUSHA_TILE 4096  // entries per slot without EdgeValue (24 KB); halved with EdgeValue (20 KB)
#endif
#ifndef CUSHA_PERSISTENT
#define CUSHA_PERSISTENT 1
#endif
#ifndef CUSHA_MIN_BLOCKS
#define CUSHA_MIN_BLOCKS 2
#endif
#ifndef CUSHA_GSU
#define CUSHA_GSU 8
#endif
constexpr int kGSU = CUSHA_GSU;  // G-Shards write-back: SrcIndex loads in flight per lane
#ifndef CUSHA_L2HINT
#define CUSHA_L2HINT 0  // 1: evict-first on topology streams; 2: also on SrcValue reads
#endif
constexpr bool kPersistent = CUSHA_PERSISTENT != 0;  // grid = resident CTAs (queue) vs one CTA per shard
#ifndef CUSHA_VB
#define CUSHA_VB 8
#endif
#ifndef CUSHA_SPEC
#define CUSHA_SPEC 1
#endif
#ifndef CUSHA_SPEC_ALWAYS
#define CUSHA_SPEC_ALWAYS 0  // 1: prefetch CW stage-4 tiles for every shard (dropped when it stays idle)
#endif
constexpr uint32_t kVB = CUSHA_VB;                   // vertex loads in flight per thread in stages 1 and 3
#ifndef CUSHA_EPT
#define CUSHA_EPT 4
#endif
constexpr uint32_t kEPT = CUSHA_EPT;  // stage-2 entries per consumer thread per step (4 or 8)
#ifndef CUSHA_PF
#define CUSHA_PF 2  // L2 prefetch of a shard's stage-3 vertex data (and delta row): 1 by the producer at ticket draw, 2 by a consumer at stage-2 start
#endif
#ifndef CUSHA_S4U
#define CUSHA_S4U 1
#endif
#ifndef CUSHA_S4TWO_ALL
#define CUSHA_S4TWO_ALL 0  // 1: the float algorithms also take 2 stage-4 entries per step at one CTA per SM
#endif
#ifndef CUSHA_S4U_INT
#define CUSHA_S4U_INT 1
#endif
// stage-4 entries per consumer thread per step (loads before stores), per
// kind of algorithm: 2 for the integer ones gained 4% on C4 SSWP but lost up
// to 7% on C3 depending on the box, 2 for PR lost 2.5% (DESIGN.md tuning log)
template <class A>
constexpr uint32_t s4u_of() {
  return A::kMonotone ? CUSHA_S4U_INT : CUSHA_S4U;
}
constexpr uint32_t kConsumerWarps = CUSHA_CONSUMER_WARPS;
constexpr uint32_t kConsumers = kConsumerWarps * 32;
#ifndef CUSHA_BK
#define CUSHA_BK 1
#endif
// 1: a bookkeeper warp does each shard's end-of-ticket bookkeeping (trace
// counters, predictor, convergence flag, ticket_done's fence and atomics) so
// that the consumer warps go straight on with the next shard
constexpr bool kBk = CUSHA_BK != 0;
#ifndef CUSHA_AHEAD
#define CUSHA_AHEAD 1  // stage-2 tiles the producer prefetches into L2 beyond the one it pushes (KParams::ahead)
#endif
#ifndef CUSHA_AHEAD_WAIT
#define CUSHA_AHEAD_WAIT 1  // the read-ahead starts before the producer's ticket_wait
#endif
#ifndef CUSHA_EARLY_SEQ
#define CUSHA_EARLY_SEQ 1  // a shard's next pass is released at the end of its ticket: 1 by the consumers, 2 by the bookkeeper warp before its bookkeeping (0: after it)
#endif
#ifndef CUSHA_DROW_ASYNC
#define CUSHA_DROW_ASYNC 1  // the stage-4 delta row arrives by cp.async during stage 2 (0: loads in stage 1)
#endif
#ifndef CUSHA_AHEAD4
#define CUSHA_AHEAD4 1  // the L2 read-ahead also covers CW stage-4 tiles
#endif
constexpr uint32_t kPassThreads = kConsumers + 32 + (kBk ? 32 : 0);  // + 1 producer warp (+ 1 bookkeeper warp)
constexpr uint32_t kBkWarp = kConsumerWarps + 1;
// one finished ticket, handed from the consumers to the bookkeeper warp
struct BkRec {
  uint32_t s, it, any, upd;
  unsigned long long stores;
};
// entries per ring slot
template <class A>
constexpr uint32_t tile_of() {
  return A::kEdge ? CUSHA_TILE / 2 : CUSHA_TILE;
}
constexpr uint32_t kStages = CUSHA_STAGES;          // ring depth (the default)
#ifndef CUSHA_MAX_STAGES
#define CUSHA_MAX_STAGES 8
#endif
// ring depth of a run (KParams::nst): kStages, or more when shared memory has
// room for another slot at the same CTAs per SM (chosen by the host)
constexpr uint32_t kMaxStages = CUSHA_MAX_STAGES > CUSHA_STAGES ? CUSHA_MAX_STAGES : CUSHA_STAGES;
constexpr uint32_t kConsumerBar = 1;                // named barrier of the consumer warps

// ring slot: stage 2 = SrcValue (4T) | DestIndex (2T) | EdgeValue (4T);
//            stage 4 = SrcIndexCW (2T) | Mapper (4T)
template <class A>
constexpr uint32_t slot_bytes() {
  return tile_of<A>() * (6 + (A::kEdge ? 4 : 0));
}
// run-start bitmap words a stage-4 slot carries (tile starts are 8-aligned;
// the 16-byte TMA copy is aligned to 128 entries)
template <class A>
constexpr uint32_t bits_words() {
  return tile_of<A>() / 32 + 8;
}
// Mapper runs (RunT - RunK, 4 B each) a stage-4 slot holds after SrcIndexCW and the bitmap
template <class A>
constexpr uint32_t run_cap() {
  return (slot_bytes<A>() - 2 * tile_of<A>() - 4 * bits_words<A>()) / 4 / 4 * 4;
}
#ifndef CUSHA_RLE
#define CUSHA_RLE 0  // measured slower (the pass is consumer-bound): DESIGN.md "Tuning log"
#endif
constexpr bool kRle = CUSHA_RLE != 0;  // stream Mapper as runs
// Mapper in window form, chosen per run
// (KParams::mapj) when the shard's delta row fits in shared memory without
// costing occupancy: a stage-4 tile then carries SrcIndexCW and the u16
// window index j of each entry (4 B per entry instead of 6 B with the u32
// Mapper), and Mapper[k] = delta_row[j] + k with the row loaded in stage 1.
// Stage-4 entries per tile: a whole slot in either form.
template <class A>
constexpr uint32_t tile4j_of() {
  return slot_bytes<A>() / 4 / 8 * 8;
}
template <class A>
constexpr uint32_t tile4m_of() {
  return kRle ? tile_of<A>() : slot_bytes<A>() / 6 / 8 * 8;
}
#ifndef CUSHA_DIAG
#define CUSHA_DIAG 0
#endif
// Diagnostic variants for the per-stage cost split (tools/diag_pass.py; never
// the product, results are wrong by design): bit 0 = every shard active in
// every pass (no convergence), bit 1 = no stage-2 reduction, bit 2 = no
// stage-4 stores, bit 3 = no per-pass trace counters (stats only).
constexpr uint32_t kDiag = CUSHA_DIAG;
#ifndef CUSHA_TIMELINE
#define CUSHA_TIMELINE 0
#endif
// Diagnostic timeline (tools/timeline.py; never the product): %globaltimer
// stamps of each ticket's steps, kTlSlots words per ticket, ticket = pass * |S|
// + shard.  0 producer drew it, 1 producer passed ticket_wait, 2 consumers got
// its first tile, 3 stage 1 done, 4 stage 2 done, 5 stage 3 done, 6 stage 4
// done, 7 ticket completed, 8 CTA index, 9 stage-4 tiles were prefetched,
// 10 first stage-4 tile acquired, 11 last stage-4 tile processed (thread 0),
// 12 thread 0 finished its stage-3 vertices (before the stage-3 barrier).
constexpr uint32_t kTlSlots = 13, kTlCap = 1u << 18;
#if CUSHA_TIMELINE
__device__ uint32_t g_timeline[kTlCap * kTlSlots];
__device__ __forceinline__ void tl_mark(uint32_t ticket, uint32_t k, uint32_t v = 0xFFFFFFFFu) {
  if (ticket >= kTlCap) return;
  if (v == 0xFFFFFFFFu) asm volatile("mov.u32 %0, %%globaltimer_lo;" : "=r"(v));
  g_timeline[ticket * kTlSlots + k] = v;
}
#else
__device__ __forceinline__ void tl_mark(uint32_t, uint32_t, uint32_t = 0) {}
#endif

// stage-4 tile kinds: kDescStage4 carries SrcIndexCW + Mapper per entry;
// kDescStage4R carries SrcIndexCW + the Mapper runs overlapping the tile.
enum : uint32_t { kDescStage2 = 0, kDescStage4 = 1, kDescDone = 2, kDescStage4R = 3 };
enum : uint32_t { kFlagLast = 1, kFlagSpec4 = 2 };
// flags: kFlagLast = last tile of this stage; kFlagSpec4 (on a shard's first
// tile) = stage-4 tiles of this shard follow its stage-2 tiles.  n = entries
// copied into the slot; [lo, hi) = the entries the consumers use; base = CW
// position of entry 0 of the slot; nruns = runs in the slot (kDescStage4R).
struct __align__(16) TileDesc {
  uint32_t shard, kind, n, flags, lo, hi, base, nruns, pass, tgt;  // tgt: partition receiving a stage-4 tile's stores
};

// ------------------------------------------------ overlapped passes (row a5)
// One launch runs every pass: shard tickets
// t = 0, 1, 2, ... are drawn from one counter (shard t % |S| of pass t / |S|),
// so a CTA that finishes its part of pass k goes on with pass k + 1 instead of
// idling at an iteration barrier: the paper's asynchronous model (L45) carried
// across the iteration boundary.  Two waits bound the overlap:
//  - pass k of shard s starts after pass k - 1 of s completed (one CTA owns a
//    shard's VertexValues at a time, as in Fig. 5);
//  - pass k starts after pass k - W completed (at most W passes in flight;
//    W = KParams::window, 2 by default, 4 for low-degree graphs).
// Convergence (L189, "a pass that commits nothing") is concluded when W
// consecutive passes k - W + 1 .. k all committed nothing.  Why that is exact:
// let T0 be the moment pass k - W completed.  Every ticket of pass k read its
// inputs after T0, and no write happens after T0 until some commit; take the
// first commit after T0, by a ticket of pass q on shard s.  Passes <= k - W
// finished writing before T0 (a shard's pass-r ticket starts after its pass
// r - 1 finished writing, so pass r complete implies every earlier pass's
// writes complete) and passes
// k - W + 1 .. k commit nothing, so q > k, and that ticket read the
// state at T0 - as did shard s's pass-k ticket, which ran between T0 and it
// and committed nothing from the same inputs and the same VertexValues
// (integer and fixed-point sums are order-independent, R11).  The same inputs
// give the same result, so no such commit exists: the state at T0 is the
// fixed point a barrier-separated pass would confirm.
__device__ __forceinline__ uint32_t ld_vol(const uint32_t* a) { return *reinterpret_cast<const volatile uint32_t*>(a); }
__device__ __forceinline__ void st_vol(uint32_t* a, uint32_t v) { *reinterpret_cast<volatile uint32_t*>(a) = v; }
__device__ __forceinline__ void fence_sc_gpu() { asm volatile("fence.sc.gpu;" ::: "memory"); }

// the producer's waits before ticket (s, pass) may read anything; false: the
// run stopped meanwhile (the ticket is abandoned - every waiting ticket polls
// stop, so an abandoned ticket never leaves another one waiting for it)
// known: every pass below it is known (to this producer) to have completed
__device__ __forceinline__ bool ticket_wait(const KParams& p, uint32_t s, uint32_t pass, uint32_t Sloc, uint32_t& known) {
  // both conditions' first reads in flight together (the common case: both hold)
  const bool need_w = pass >= p.window && pass - p.window >= known;
  const uint32_t seq0 = ld_vol(&p.shard_seq[s]);
  const uint32_t done0 = need_w ? ld_vol(&p.trace[pass - p.window].done) : Sloc;
  if (seq0 >= pass && done0 >= Sloc) {
    if (need_w) known = pass - p.window + 1;
    __threadfence();                                      // acquire the completed passes' stores ...
    asm volatile("fence.proxy.async.global;" ::: "memory");  // ... for the TMA (async-proxy) reads too
    return true;
  }
  while (ld_vol(&p.shard_seq[s]) < pass) {
    if (ld_vol(&p.ctl->stop)) return false;
    __nanosleep(64);
  }
  if (pass >= p.window && pass - p.window >= known) {
    while (ld_vol(&p.trace[pass - p.window].done) < Sloc) {
      if (ld_vol(&p.ctl->stop)) return false;
      __nanosleep(64);
    }
    known = pass - p.window + 1;  // pass r complete implies every earlier pass complete
  }
  __threadfence();                                      // acquire the completed passes' stores ...
  asm volatile("fence.proxy.async.global;" ::: "memory");  // ... for the TMA (async-proxy) reads too
  return true;
}

// ticket (s, pass) finished (its stores ordered before by the caller's
// barrier; fences are cumulative).  The thread completing the last ticket of
// a clean pass looks at both neighbouring passes.
__device__ __forceinline__ void ticket_done(const KParams& p, uint32_t s, uint32_t pass, uint32_t Sloc,
                                            bool set_seq = true) {
  __threadfence();
  if (set_seq) st_vol(&p.shard_seq[s], pass + 1);
  if (atomicAdd(&p.trace[pass].done, 1u) != Sloc - 1) return;
  fence_sc_gpu();  // pairs with the other neighbour's completer: at least one of two sees both complete
  if (ld_vol(&p.trace[pass].active_shards) != 0) return;
  auto clean = [&](uint32_t r) {
    if (ld_vol(&p.trace[r].done) != Sloc) return false;
    __threadfence();  // acquire: the completers' active_shards increments precede their done increments
    return ld_vol(&p.trace[r].active_shards) == 0;
  };
  // W consecutive clean passes, one of them this one: a window [a, a + W) containing pass
  const uint32_t W = p.window;
  uint32_t conv = 0xFFFFFFFFu;
  for (uint32_t a = pass + 1 > W ? pass + 1 - W : 0u; a <= pass && conv == 0xFFFFFFFFu; ++a) {
    if (a + W > p.ctl->max_iters) break;
    bool ok = true;
    for (uint32_t r = a; r < a + W && ok; ++r)
      if (r != pass) ok = clean(r);
    if (ok) conv = a + W;
  }
  if (conv != 0xFFFFFFFFu) {
    atomicMin(&p.ctl->conv_iter, conv);
    st_vol(&p.ctl->stop, 1u);
  }
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

template <class A>
__device__ __forceinline__ void proc8(uint32_t* sm, uint32_t st, const uint4& s0, const uint4& s1, const uint4& dd,
                                      const uint4& e0, const uint4& e1) {
  const uint32_t D[8] = {dd.x & 0xFFFFu, dd.x >> 16, dd.y & 0xFFFFu, dd.y >> 16,
                         dd.z & 0xFFFFu, dd.z >> 16, dd.w & 0xFFFFu, dd.w >> 16};
  const uint32_t S[8] = {s0.x, s0.y, s0.z, s0.w, s1.x, s1.y, s1.z, s1.w};
  const uint32_t W[8] = {e0.x, e0.y, e0.z, e0.w, e1.x, e1.y, e1.z, e1.w};
  if constexpr (A::kAcc == 0) {
#pragma unroll
    for (int k = 0; k < 8; ++k) A::compute(sm, st, D[k], S[k], W[k]);
  } else {
    uint64_t F[8][2];
#pragma unroll
    for (int k = 0; k < 8; ++k) A::contrib(sm, st, D[k], S[k], W[k], F[k]);
    uint32_t old[8][2];
#pragma unroll
    for (int k = 0; k < 8; ++k)
#pragma unroll
      for (int a = 0; a < A::kAcc; ++a) old[k][a] = atomicAdd(&sm[A::acc_lo(a) * st + D[k]], (uint32_t)F[k][a]);
#pragma unroll
    for (int k = 0; k < 8; ++k)
#pragma unroll
      for (int a = 0; a < A::kAcc; ++a) {
        const uint32_t l = (uint32_t)F[k][a];
        const uint32_t h = (uint32_t)(F[k][a] >> 32) + ((old[k][a] + l < old[k][a]) ? 1u : 0u);
        if (h) atomicAdd(&sm[(A::acc_lo(a) + 1) * st + D[k]], h);
      }
  }
}

// stage-4 value of local vertex l and whether it must be stored
// wbs (integer algorithms with the stage-1 stash): after stage 3 the stash
// holds each vertex's new value, or A::kNoWb when it did not change - one
// shared load per entry instead of the changed bit and the value
template <class A>
__device__ __forceinline__ bool wb_get(const uint32_t* sm, const uint32_t* aux, const uint32_t* wbs, uint32_t l,
                                       uint32_t& val) {
  if constexpr (A::kMonotone) {
    // integer algorithms: local == committed value whenever not updated, so
    // copies of unchanged vertices already hold it (R19) — store only changed
    if (wbs) {
      val = wbs[l];
      return val != A::kNoWb;
    }
    if (!((aux[l >> 5] >> (l & 31)) & 1u)) return false;
    val = sm[l];
    return true;
  } else {
    val = aux[l];  // local_vertices as left by update_condition (Fig. 5 line 25)
    return true;
  }
}

// ------------------------------------------------- G-Shards window walker
// Visits every entry of the windows W_sj (j = 0..S-1) of source shard s:
// each warp takes 32 windows at a time, scans their lengths across lanes and
// walks the concatenation with one entry per lane (kGSU in flight), finding
// each entry's window by a 5-step binary search over the lanes' prefix sums.
// The next batch's window bounds are loaded while the current one is walked.
// fn(e, l): e = shard position, l = SrcIndex - s*N.
template <class Fn>
__device__ __forceinline__ void gs_walk(const KParams& p, uint32_t s, uint32_t lane, uint32_t warp, uint32_t nwarps,
                                        Fn&& fn) {
  const uint32_t* r0 = p.win + (size_t)s * p.S;
  const uint32_t* r1 = r0 + p.S;
  uint32_t na = 0, nb = 0;
  if (warp * 32 + lane < p.S) { na = __ldg(r0 + warp * 32 + lane); nb = __ldg(r1 + warp * 32 + lane); }
  for (uint32_t jb = warp * 32; jb < p.S; jb += nwarps * 32) {
    const uint32_t a = na, b = nb;
    const uint32_t jn = jb + nwarps * 32 + lane;
    na = nb = 0;
    if (jn < p.S) { na = __ldg(r0 + jn); nb = __ldg(r1 + jn); }
    const uint32_t len = b - a;
    uint32_t inc = len;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t t = __shfl_up_sync(kFull, inc, o);
      if (lane >= (uint32_t)o) inc += t;
    }
    const uint32_t total = __shfl_sync(kFull, inc, 31);
    const uint32_t exc = inc - len;
    for (uint32_t f0 = 0; f0 < total; f0 += 32 * kGSU) {
      uint32_t e[kGSU], l[kGSU];
#pragma unroll
      for (int u = 0; u < kGSU; ++u) {
        const uint32_t f = f0 + u * 32 + lane;
        int w = 0;
#pragma unroll
        for (int step = 16; step; step >>= 1) {
          const uint32_t ex = __shfl_sync(kFull, exc, w + step);
          if (ex <= f) w += step;
        }
        e[u] = __shfl_sync(kFull, a, w) + (f - __shfl_sync(kFull, exc, w));
        l[u] = f < total ? (uint32_t)__ldg(topo_at(p.srcloc, p.srcloc_h, p.splitP, e[u])) : 0xFFFFFFFFu;
      }
#pragma unroll
      for (int u = 0; u < kGSU; ++u)
        if (l[u] != 0xFFFFFFFFu) fn(e[u], l[u]);
    }
  }
}

// ------------------------------------------------------------ producer
// Per shard: its stage-2 tiles, then — for CW — its stage-4 tiles, either
// right away (shard predicted active: prefetch overlaps stage 3) or once the
// consumers' stage 3 has decided values_updated (decide_bar / s_any).
// Stage-4 tiles are cut per target partition q (CW_s lists W_s0, W_s1, ... in
// j order, L175, and partitions are contiguous j ranges, so the entries aimed
// at partition q are one contiguous segment): a tile's stores all go to
// sv_peer[q], the partition that owns its windows (one segment on one GPU).
template <class A, int REPR>
__device__ __forceinline__ void producer(const KParams& p, uint8_t* ring, TileDesc* desc, uint64_t* full_bar,
                                         uint64_t* empty_bar, uint64_t* decide_bar, const volatile int* s_any) {
  constexpr uint32_t SLOT = slot_bytes<A>();
  constexpr uint32_t kTile = tile_of<A>();
  constexpr uint32_t kRunCap = run_cap<A>();
  uint32_t slot = 0, ph = 0, dph = 0, cur_pass = 0;
  const uint64_t pol = l2_evict_first_policy();
  auto push = [&](uint32_t shard, uint32_t kind, uint32_t n, uint32_t flags, const void* g0, uint32_t b0,
                  const void* g1, uint32_t o1, uint32_t b1, const void* g2, uint32_t o2, uint32_t b2,
                  uint32_t lo = 0, uint32_t hi = 0xFFFFFFFFu, uint32_t base = 0, uint32_t nruns = 0,
                  const void* g3 = nullptr, uint32_t o3 = 0, uint32_t b3 = 0, uint32_t tgt = 0) {
    mbar_wait(&empty_bar[slot], ph ^ 1);
    desc[slot] = TileDesc{shard, kind, n, flags, lo, hi == 0xFFFFFFFFu ? n : hi, base, nruns, cur_pass, tgt};
    uint8_t* buf = ring + slot * SLOT;
    const uint32_t bytes = b0 + b1 + b2 + b3;
    if (bytes) {
      mbar_expect_tx(&full_bar[slot], bytes);
      if (b3) bulk_g2s(buf + o3, g3, b3, &full_bar[slot]);
      // topology streams (DestIndex, EdgeValue, SrcIndexCW, Mapper) are read once per
      // pass: evict-first; SrcValue (g0 of a stage-2 tile) keeps the default policy
      const bool sv = kind == kDescStage2;
      if (b0) {
        if (CUSHA_L2HINT >= (sv ? 2 : 1)) bulk_g2s_hint(buf, g0, b0, &full_bar[slot], pol);
        else bulk_g2s(buf, g0, b0, &full_bar[slot]);
      }
      if (b1) {
        if (CUSHA_L2HINT >= 1) bulk_g2s_hint(buf + o1, g1, b1, &full_bar[slot], pol);
        else bulk_g2s(buf + o1, g1, b1, &full_bar[slot]);
      }
      if (b2) {
        if (CUSHA_L2HINT >= 1) bulk_g2s_hint(buf + o2, g2, b2, &full_bar[slot], pol);
        else bulk_g2s(buf + o2, g2, b2, &full_bar[slot]);
      }
    } else {
      mbar_arrive(&full_bar[slot]);
    }
    if (++slot == p.nst) { slot = 0; ph ^= 1; }
  };
  const uint32_t Sloc = p.Sl;
  // L2 prefetch of stage-2 tile [t0, t0 + kTile) of a shard ending at e (device-resident parts only)
  auto pf2 = [&](uint32_t t0, uint32_t e) {
    if (t0 >= e) return;
    const uint32_t n = min(kTile, e - t0);
    bulk_prefetch_l2(p.srcvalue + t0, n * 4);
    if (t0 + n <= p.splitP) {
      bulk_prefetch_l2(p.dest + t0, n * 2);
      if (A::kEdge) bulk_prefetch_l2(p.ev + t0, n * 4);
    }
  };
  // L2 prefetch of the CW stage-4 tile at CW position k0 (< ke), device-resident parts only
  auto pf4 = [&](uint32_t k0, uint32_t ke) {
    if (k0 >= ke || k0 >= p.splitQ) return;
    const uint32_t n = min(p.mapj ? tile4j_of<A>() : tile4m_of<A>(), ke - k0);
    bulk_prefetch_l2(p.cw_src + k0, n * 2);
    if (p.mapj) bulk_prefetch_l2(p.cw_win + k0, n * 2);
    else bulk_prefetch_l2(p.mapper + k0, n * 4);
  };
  // CW_s's segment aimed at partition q: [*a, *b)
  auto segment = [&](uint32_t s, uint32_t q, uint32_t* a, uint32_t* b) {
    if (p.G > 1) {
      const uint32_t* row = p.cwp + (size_t)s * (p.G + 1);
      *a = row[q];
      *b = row[q + 1];
    } else {
      *a = p.cw_off[s];
      *b = *a + p.cw_cnt[s];
    }
  };
  // tiles prefetched into L2 beyond the ring, when the pass streams from HBM (KParams::ahead)
  const uint32_t ahead = p.ahead ? CUSHA_AHEAD : 0u;
  const uint32_t max_iters = p.ctl->max_iters;  // constant during the launch
  uint32_t known_done = 0;                      // passes below it have completed (ticket_wait)
  for (uint32_t round = 0;; ++round) {
    uint32_t s;  // local shard index
    uint32_t sb = 0, se = 0;  // the shard's entry range (read before the waits in overlapped mode)
    uint32_t ca = 0, cb = 0;  // one partition: CW_s = [ca, cb) (read with them)
    uint8_t act = 0;          // stage-4 predictor (a hint: a stale read costs bandwidth, not correctness)
    if (p.multi) {
      // overlapped passes: the next ticket, whatever pass it belongs to
      const unsigned long long t = atomicAdd(&p.ctl->ticket, 1ull);
      cur_pass = (uint32_t)(t / Sloc);
      s = (uint32_t)(t - (unsigned long long)cur_pass * Sloc);
      if (p.order && cur_pass < max_iters) s = p.order[s];
      bool over = cur_pass >= max_iters || ld_vol(&p.ctl->stop) != 0;
      if (CUSHA_TIMELINE && !over) tl_mark((uint32_t)t, 0);
      if (!over) {
        // the shard's scalars and first stage-2 tiles start towards the SM / L2
        // while the producer waits (a prefetch reads nothing into the CTA, so it
        // needs no ordering; the offsets are read-only)
        sb = p.shard_off[s];
        se = p.shard_off[s + 1];
        act = p.active[s];
        if (REPR == CUSHA_REPR_CW && p.G == 1) {
          ca = p.cw_off[s];
          cb = ca + p.cw_cnt[s];
        }
        if (CUSHA_AHEAD_WAIT && ahead)
          for (uint32_t j = 0; j <= ahead; ++j) pf2(sb + j * kTile, se);
        over = !ticket_wait(p, s, cur_pass, Sloc, known_done);
      }
      if (over) {
        push(0, kDescDone, 0, 0, nullptr, 0, nullptr, 0, 0, nullptr, 0, 0);
        return;
      }
      if (CUSHA_TIMELINE) tl_mark(cur_pass * Sloc + s, 1);
    } else {
      // persistent grid: shards from the global queue; otherwise CTA b runs shard b only
      s = kPersistent ? atomicAdd(&p.ctl->next_shard, 1u) : (round == 0 ? blockIdx.x : Sloc);
      if (p.order && s < Sloc) s = p.order[s];
      if (s >= Sloc) {
        push(0, kDescDone, 0, 0, nullptr, 0, nullptr, 0, 0, nullptr, 0, 0);
        return;
      }
    }
    if (p.skip) {
      // clean-shard skipping (opt-in): no
      // window of shard s was written since its last pass, so stages 1-3 would
      // recompute the values it already holds and commit nothing.  Clearing the
      // flag before the tiles are read means a write landing after this point
      // re-marks s for a later pass.
      if (atomicExch(&p.dirty[s], 0u) == 0u) {
        p.active[s] = 0;
        if (p.multi) ticket_done(p, s, cur_pass, Sloc);
        continue;
      }
      __threadfence();                                      // acquire the writers' SrcValue stores ...
      asm volatile("fence.proxy.async.global;" ::: "memory");  // ... for the TMA (async-proxy) reads below
    }
    if (!p.multi) {
      sb = p.shard_off[s];
      se = p.shard_off[s + 1];
      act = p.active[s];
      if (REPR == CUSHA_REPR_CW && p.G == 1) {
        ca = p.cw_off[s];
        cb = ca + p.cw_cnt[s];
      }
    }
    const bool spec = CUSHA_SPEC && REPR == CUSHA_REPR_CW && (CUSHA_SPEC_ALWAYS || act);
    const uint32_t b = sb, e = se;
    if (CUSHA_PF == 1) {
      // the consumers' global reads of this shard (stage 1/3 VertexValues and
      // NbrsNum, the stage-4 delta row) become L2 hits: one TMA prefetch each
      const uint32_t off = s * p.N, nv = min(p.N, p.V - (p.s0 + s) * p.N);
      bulk_prefetch_l2(reinterpret_cast<const typename A::Value*>(p.vv) + off, nv * (uint32_t)sizeof(typename A::Value));
      if (A::kOutDeg) bulk_prefetch_l2(p.outdeg + off, nv * 4);
      if (REPR == CUSHA_REPR_CW && p.mapj) bulk_prefetch_l2(p.cw_delta + (size_t)s * p.S, p.S * 4);
    }
    // first / last non-empty stage-4 segment of CW_s (stage-4 tiles are 8-entry aligned for TMA)
    uint32_t qa = 0, qz = 0, a0 = 0, b0 = 0;
    if (REPR == CUSHA_REPR_CW) {
      for (uint32_t q = 0; q < p.G; ++q) {
        uint32_t x = ca, y = cb;
        if (p.G > 1) segment(s, q, &x, &y);
        if (x < y) {
          if (qz == 0) { qa = q; a0 = x; }
          qz = q + 1;
          b0 = y;
        }
      }
    }
    if (b == e) push(s, kDescStage2, 0, kFlagLast | (spec ? kFlagSpec4 : 0u), nullptr, 0, nullptr, 0, 0, nullptr, 0, 0);
    if (!(CUSHA_AHEAD_WAIT && p.multi))
      for (uint32_t j = 1; j <= ahead; ++j) pf2(b + j * kTile, e);
    for (uint32_t t0 = b; t0 < e; t0 += kTile) {
      const uint32_t n = min(kTile, e - t0);
      const uint32_t flags = (t0 + n >= e ? kFlagLast : 0u) | (t0 == b && spec ? kFlagSpec4 : 0u);
      push(s, kDescStage2, n, flags, p.srcvalue + t0, n * 4, topo_at(p.dest, p.dest_h, p.splitP, t0), 4 * kTile,
           n * 2, A::kEdge ? (const void*)topo_at(p.ev, p.ev_h, p.splitP, t0) : nullptr, 6 * kTile,
           A::kEdge ? n * 4 : 0u);
      if (ahead) {
        if (t0 + (ahead + 1) * kTile < e) pf2(t0 + (ahead + 1) * kTile, e);
        else if (CUSHA_AHEAD4 && spec && t0 + kTile >= e && qz) pf4(a0 & ~7u, (b0 + 7u) & ~7u);  // the first stage-4 tile
      }
    }
    bool send4 = spec;
    if (REPR == CUSHA_REPR_CW && !spec) {
      mbar_wait(decide_bar, dph);  // consumers finished stage 3 of shard s
      dph ^= 1;
      send4 = *s_any != 0;
    }
    if (send4) {
      // [lo, hi) marks the valid part of each tile
      const uint32_t kT4 = p.mapj ? tile4j_of<A>() : tile4m_of<A>();
      if (qz == 0) push(s, kDescStage4, 0, kFlagLast, nullptr, 0, nullptr, 0, 0, nullptr, 0, 0);
      for (uint32_t q = qa; q < qz; ++q) {
        uint32_t a, b2;
        segment(s, q, &a, &b2);
        if (a >= b2) continue;
        const uint32_t kb = a & ~7u, ke = (b2 + 7u) & ~7u;
        for (uint32_t k0 = kb; k0 < ke; k0 += kT4) {
          const uint32_t n = min(kT4, ke - k0);
          const uint32_t fl = (k0 + n >= ke && q + 1 == qz) ? kFlagLast : 0u, lo = a > k0 ? a - k0 : 0u,
                         hi = min(b2 - k0, n);
          if (kRle) {
            // runs from the one containing position k0/128*128 (the slot's first
            // bitmap position) through the last starting inside the tile; the
            // TMA copy starts 4-aligned, so that run sits at list index ra - ra4
            const uint32_t ra = p.run_unit[k0 / kRunUnit];
            const uint32_t rb = min(p.R, p.run_unit[(k0 + n - 1) / kRunUnit + 1] + 1);
            const uint32_t ra4 = ra & ~3u, nr = ((rb + 3u) & ~3u) - ra4;
            if (nr <= kRunCap) {
              // slot: SrcIndexCW | RunT-RunK per run | run-start bitmap words [k0/128*4, ceil((k0+n)/128)*4)
              const uint32_t wa = k0 / 128 * 4, wz = (k0 + n + 127) / 128 * 4;
              push(s, kDescStage4R, n, fl | ((ra - ra4) << 8), topo_at(p.cw_src, p.cw_src_h, p.splitQ, k0), n * 2,
                   p.run_d + ra4, 2 * kTile,
                   nr * 4, p.run_bits + wa, 2 * kTile + 4 * kRunCap, (wz - wa) * 4, lo, hi, k0, nr, nullptr, 0, 0, q);
              continue;
            }
          }
          if (p.mapj)
            push(s, kDescStage4, n, fl, topo_at(p.cw_src, p.cw_src_h, p.splitQ, k0), n * 2,
                 topo_at(p.cw_win, p.cw_win_h, p.splitQ, k0), 2 * kT4, n * 2, nullptr, 0, 0, lo, hi, k0, 0,
                 nullptr, 0, 0, q);
          else
            push(s, kDescStage4, n, fl, topo_at(p.cw_src, p.cw_src_h, p.splitQ, k0), n * 2,
                 topo_at(p.mapper, p.mapper_h, p.splitQ, k0), 2 * kT4, n * 4, nullptr, 0, 0, lo, hi, k0, 0,
                 nullptr, 0, 0, q);
          if (CUSHA_AHEAD4 && ahead) pf4(k0 + kT4, ke);
        }
      }
    }
  }
}

// end-of-ticket bookkeeping of shard s in pass it: trace counters, the
// stage-4 predictor, the paper's is_converged = false (line 26), and - with
// overlapped passes - the ticket's completion (ticket_done)
__device__ __forceinline__ void ticket_bookkeeping(const KParams& p, uint32_t s, uint32_t it, bool any, uint32_t upd,
                                                   unsigned long long stores, uint32_t Sloc) {
  if (it < p.trace_cap && !(kDiag & 8)) {
    atomicAdd(&p.trace[it].edges, (unsigned long long)p.shard_cnt[s]);
    atomicAdd(&p.trace[it].shards, 1ull);
  }
  p.active[s] = any ? 1 : 0;
  if (any) {
    *reinterpret_cast<volatile uint32_t*>(&p.ctl->changed) = 1u;
    if (it < p.trace_cap) {
      TraceRec* t = p.trace + it;
      atomicAdd(&t->active_shards, 1u);  // read by the convergence test (ticket_done)
      if (!(kDiag & 8)) {
        atomicAdd(&t->updated, upd);
        atomicAdd(&t->wb_entries, (unsigned long long)p.cw_cnt[s]);
        atomicAdd(&t->wb_stores, stores);
      }
    }
  }
  // overlapped passes: every consumer's stores precede this (barriers; fences are cumulative);
  // with CUSHA_EARLY_SEQ the consumers released the shard's next pass already
  if (p.multi) ticket_done(p, s, it, Sloc, !(CUSHA_EARLY_SEQ && kBk));
}

template <class A, int REPR>
__global__ void __launch_bounds__(kPassThreads, CUSHA_MIN_BLOCKS) shard_pass(const KParams p) {
  extern __shared__ __align__(128) uint8_t dyn[];
  constexpr uint32_t SLOT = slot_bytes<A>();
  constexpr uint32_t kTile = tile_of<A>();
  uint8_t* const ring = dyn;
  const uint32_t nst = p.nst;
  uint32_t* const sm = reinterpret_cast<uint32_t*>(dyn + nst * SLOT);
  __shared__ uint64_t full_bar[kMaxStages], empty_bar[kMaxStages], decide_bar;
  __shared__ TileDesc desc[kMaxStages];
  __shared__ uint32_t s_upd;
  __shared__ int s_any;
  __shared__ unsigned long long s_stores;
  __shared__ uint64_t bk_full[2], bk_empty[2];
  __shared__ BkRec bk[2];
  using V_t = typename A::Value;
  const uint32_t tid = threadIdx.x, lane = tid & 31u, warp = tid >> 5;
  const uint32_t N = p.N, st = N + 1;
  // aux: the changed bits of stage 3 (integer algorithms), or the write-back
  // values of local_vertices (float algorithms), which stage 3 stores over the
  // first fixed-point word of the same vertex: its sum is dead once read
  uint32_t* const tail = sm + A::kWords * st;
  uint32_t* const aux = A::kMonotone ? tail : sm + A::acc_lo(0) * st;
  // Mapper-delta row of the current shard (window form, p.mapj)
  uint32_t* const drow = tail + (A::kMonotone ? (N + 31) / 32 : 0);
  // stage 1's VertexValues of the shard, for stage 3 (integer algorithms, p.stash)
  uint32_t* const stash = drow + (p.mapj ? p.S : 0u);
  const uint32_t* const wbs = (A::kMonotone && p.stash) ? stash : nullptr;
  constexpr uint32_t kS4U = s4u_of<A>();
  const uint32_t it0 = *reinterpret_cast<volatile uint32_t*>(&p.ctl->iter);
  // a pass launched after the run converged / hit max_iters is a no-op (host-loop mode)
  if (*reinterpret_cast<volatile uint32_t*>(&p.ctl->converged) || it0 >= p.ctl->max_iters) return;
  const uint32_t Sloc = p.Sl;
  if (tid == 0) {
    for (uint32_t i = 0; i < nst; ++i) {
      mbar_init(&full_bar[i], 1);                // the producer's arrive(.expect_tx)
      mbar_init(&empty_bar[i], kConsumerWarps);  // one arrive per consumer warp
    }
    mbar_init(&decide_bar, 1);  // stage-3 decision of a non-prefetched CW shard
    for (uint32_t i = 0; i < 2; ++i) {
      mbar_init(&bk_full[i], 1);   // the consumers' hand-over of a finished ticket
      mbar_init(&bk_empty[i], 1);  // the bookkeeper is done with it
    }
    mbar_fence_init();
  }
  __syncthreads();

  if (warp == 0) {
    if (lane == 0) producer<A, REPR>(p, ring, desc, full_bar, empty_bar, &decide_bar, &s_any);
  } else if (warp <= kConsumerWarps) {
    const uint32_t ct = tid - 32, cwarp = warp - 1;  // consumer thread / warp index
    uint32_t slot = 0, ph = 0;
    uint32_t ntk = 0;  // tickets handed to the bookkeeper (kBk)
    for (;;) {
      mbar_wait(&full_bar[slot], ph);
      TileDesc d = desc[slot];
      if (d.kind == kDescDone) break;
      const uint32_t s = d.shard;                  // local shard index (global p.s0 + s)
      const uint32_t it = p.multi ? d.pass : it0;  // the pass this shard belongs to
      const bool spec4 = d.flags & kFlagSpec4;
      const uint32_t off = s * N;                  // local vertex offset of the shard
      const uint32_t nv = min(N, p.V - (p.s0 + s) * N);
      V_t* vv = reinterpret_cast<V_t*>(p.vv) + off;
      const uint32_t tk = it * Sloc + s;            // timeline ticket
      if (CUSHA_TIMELINE && ct == 0) { tl_mark(tk, 2); tl_mark(tk, 8, blockIdx.x); tl_mark(tk, 9, spec4 ? 1u : 0u); }

      // ---- stage 1: local_vertices <- init_compute(VertexValues) (Fig. 5 lines 8-10, L267)
      // (kVB loads in flight per thread before any is used)
      for (uint32_t base = 0; base < nv; base += kVB * kConsumers) {
        V_t x[kVB];
#pragma unroll
        for (uint32_t u = 0; u < kVB; ++u) {
          const uint32_t v = base + u * kConsumers + ct;
          x[u] = V_t{};
          if (A::kInitReadsV && v < nv) x[u] = vv[v];
        }
#pragma unroll
        for (uint32_t u = 0; u < kVB; ++u) {
          const uint32_t v = base + u * kConsumers + ct;
          if (v < nv) {
            A::init(sm, st, v, x[u]);
            if constexpr (A::kMonotone) if (p.stash) stash[v] = x[u];
          }
        }
      }
      if (p.mapj) {  // the shard's Mapper-delta row for stage 4 (window form)
        const uint32_t* dg = p.cw_delta + (size_t)s * p.S;
        if (CUSHA_DROW_ASYNC) {
          // asynchronous copies (LDGSTS), waited for before stage 4: their latency hides behind stage 2
          for (uint32_t j = ct; j < p.S; j += kConsumers) cp_async4(drow + j, dg + j);
          cp_async_commit();
        } else {
          for (uint32_t j = ct; j < p.S; j += kConsumers) drow[j] = __ldg(dg + j);
        }
      }
      if (ct == 0) {
        A::init(sm, st, N, V_t{});  // trash slot for filler entries
        s_upd = 0;
        s_stores = 0;
      }
      bar_sync(kConsumerBar, kConsumers);
      if (CUSHA_TIMELINE && ct == 0) tl_mark(tk, 3);

      // ---- stage 2: the shard's entries from the ring, compute() into shared memory (lines 12-13, L269)
      if (CUSHA_PF == 2 && ct == 0) {
        bulk_prefetch_l2(vv, nv * (uint32_t)sizeof(V_t));
        if (A::kOutDeg) bulk_prefetch_l2(p.outdeg + off, nv * 4);
      }
      for (;;) {
        const uint8_t* buf = ring + slot * SLOT;
        if (kEPT == 8) {
          for (uint32_t i = ct * 8; i < d.n; i += kConsumers * 8) {  // n is a multiple of 8
            const uint4 sv0 = *reinterpret_cast<const uint4*>(buf + 4 * i);
            const uint4 sv1 = *reinterpret_cast<const uint4*>(buf + 4 * i + 16);
            const uint4 dd = *reinterpret_cast<const uint4*>(buf + 4 * kTile + 2 * i);
            uint4 ev0 = make_uint4(0, 0, 0, 0), ev1 = ev0;
            if (A::kEdge) {
              ev0 = *reinterpret_cast<const uint4*>(buf + 6 * kTile + 4 * i);
              ev1 = *reinterpret_cast<const uint4*>(buf + 6 * kTile + 4 * i + 16);
            }
            proc8<A>(sm, st, sv0, sv1, dd, ev0, ev1);
          }
        } else
        for (uint32_t i = ct * 4; i < d.n; i += kConsumers * 4) {
          const uint4 sv = *reinterpret_cast<const uint4*>(buf + 4 * i);
          const uint2 dd = *reinterpret_cast<const uint2*>(buf + 4 * kTile + 2 * i);
          uint4 ev = make_uint4(0, 0, 0, 0);
          if (A::kEdge) ev = *reinterpret_cast<const uint4*>(buf + 6 * kTile + 4 * i);
          if (kDiag & 2) {
            if ((sv.x ^ sv.y ^ sv.z ^ sv.w ^ dd.x ^ dd.y ^ ev.x) == 0x9e3779b9u) sm[N] = 1u;  // keep the loads
          } else {
            proc4<A>(sm, st, sv, dd, ev);
          }
        }
        __syncwarp();
        if (lane == 0) mbar_arrive(&empty_bar[slot]);
        if (++slot == nst) { slot = 0; ph ^= 1; }
        if (d.flags & kFlagLast) break;
        mbar_wait(&full_bar[slot], ph);
        d = desc[slot];
      }
      bar_sync(kConsumerBar, kConsumers);
      if (CUSHA_TIMELINE && ct == 0) tl_mark(tk, 4);

      // ---- stage 3: update_condition, commit to VertexValues, values_updated (lines 15-20, L271)
      uint32_t my_upd = 0, my_cnt = 0;
      for (uint32_t base = 0; base < nv; base += kVB * kConsumers) {
        V_t x[kVB];
        uint32_t od[kVB];
#pragma unroll
        for (uint32_t u = 0; u < kVB; ++u) {
          const uint32_t v = base + u * kConsumers + ct;
          od[u] = 0;
          if (v < nv) {
            if constexpr (A::kMonotone) x[u] = p.stash ? stash[v] : vv[v];
            else x[u] = vv[v];
            if (A::kOutDeg) od[u] = __ldg(p.outdeg + off + v);
          }
        }
#pragma unroll
        for (uint32_t u = 0; u < kVB; ++u) {
          const uint32_t v = base + u * kConsumers + ct;
          bool up = false;
          if (v < nv) {
            V_t out;
            uint32_t wbv = 0;
            up = A::update(sm, st, v, x[u], &out, &wbv, od[u]);
            if (up) vv[v] = out;
            if constexpr (A::kMonotone) {
              if (p.stash) stash[v] = up ? out : A::kNoWb;  // stage 4's write-back array (wbs)
            } else {
              aux[v] = wbv;
            }
          }
          const uint32_t m = __ballot_sync(kFull, up);
          my_cnt += __popc(m);  // (lane 0's count is the warp's; one shared atomic per warp below)
          const uint32_t w0 = base + u * kConsumers + cwarp * 32;
          if (A::kMonotone && lane == 0 && w0 < nv) aux[w0 >> 5] = m;
          my_upd |= up ? 1u : 0u;
        }
      }
      if (lane == 0 && my_cnt) atomicAdd(&s_upd, my_cnt);
      if (CUSHA_TIMELINE && ct == 0) tl_mark(tk, 12);
      // this thread's delta-row copies (issued in stage 1) land before the
      // barrier, so after it every thread sees the whole row (stage 4)
      if (CUSHA_DROW_ASYNC && p.mapj) cp_async_wait_all();
      const int any = bar_sync_or(kConsumerBar, kConsumers, (int)my_upd) | ((kDiag & 1) ? 1 : 0);
      if (CUSHA_TIMELINE && ct == 0) tl_mark(tk, 5);

      // ---- stage 4: write-back into every shard's window (lines 23-26, L308)
      uint32_t stores = 0;

      if (REPR == CUSHA_REPR_CW) {
        // thread per CW_s entry: SrcValue[Mapper[k]] = local[SrcIndex[k]] (L177, Fig. 4b);
        // consecutive threads take consecutive entries, so the stores of one
        // window (consecutive Mapper targets) coalesce into whole sectors
        if (!spec4 && ct == 0) {  // tell the producer whether CW_s's tiles are needed
          s_any = any;
          mbar_arrive(&decide_bar);
        }
        if (spec4 || any) {
          for (bool first4 = true;; first4 = false) {
            mbar_wait(&full_bar[slot], ph);
            if (CUSHA_TIMELINE && ct == 0 && first4) tl_mark(tk, 10);
            d = desc[slot];
            // the partition owning this tile's windows (this one on a single GPU):
            // in the multi-GPU mode the stores below go over NVLink to its SrcValue
            uint32_t* const svq = p.G > 1 ? p.sv_peer[d.tgt] : p.sv_write;
            if (any && d.kind == kDescStage4R) {
              // Mapper from runs: target(k) = k + D[r], D = RunT - RunK, for the run r
              // containing CW position k.  Runs start where the run-start bitmap has
              // a 1.  List entry (flags >> 8) is the run containing P = the slot's
              // first bitmap position, so for x >= P the run of position x - 1 is
              // that index + popc(bits in [P, x)) - bit(P).  Each warp takes a
              // contiguous block of 32-aligned strips, seeds its count with one
              // warp-wide popcount reduction, and lane i adds popc(word & bits <= i).
              const uint16_t* L = reinterpret_cast<const uint16_t*>(ring + slot * SLOT);
              const uint32_t* D = reinterpret_cast<const uint32_t*>(ring + slot * SLOT + 2 * kTile);
              const uint32_t* BW = D + run_cap<A>();
              const uint32_t wbase = d.base / 128 * 4;                  // word index of BW[0]
              const uint32_t alo = d.base + d.lo, ahi = d.base + d.hi;  // valid CW positions
              const uint32_t first = alo & ~31u;
              const uint32_t nstrips = (ahi - first + 31) / 32;
              const uint32_t per = (nstrips + kConsumerWarps - 1) / kConsumerWarps;
              const uint32_t s0 = first + cwarp * per * 32;
              const uint32_t s1 = min(first + (cwarp + 1) * per * 32, ahi);
              if (s0 < s1) {
                const uint32_t nw = s0 / 32 - wbase;  // bitmap words before the warp's block
                uint32_t c = 0;
                for (uint32_t w = lane; w < nw; w += 32) c += __popc(BW[w]);
                c = __reduce_add_sync(kFull, c);
                int r = (int)((d.flags >> 8) & 3u) + (int)c - (int)(BW[0] & 1u);  // run of position s0 - 1
                const uint32_t below = (2u << lane) - 1u;                          // bits 0..lane
#pragma unroll 4
                for (uint32_t sp = s0; sp < s1; sp += 32) {
                  const uint32_t word = BW[sp / 32 - wbase];
                  const int ri = r + __popc(word & below);
                  const uint32_t k = sp + lane;
                  uint32_t val;
                  if (k >= alo && k < ahi && wb_get<A>(sm, aux, wbs, L[k - d.base], val)) {
                    st_u32(svq + (k + D[ri]), val);
                    ++stores;
                  }
                  r += __popc(word);
                }
              }
            } else if (any && p.mapj) {
              // SrcValue[delta_row[j] + k] = local[SrcIndexCW[k]] for CW position k = base + i;
              // kS4U entries per thread: every shared load of a step before its stores
              const uint16_t* L = reinterpret_cast<const uint16_t*>(ring + slot * SLOT);
              const uint16_t* J = reinterpret_cast<const uint16_t*>(ring + slot * SLOT + 2 * tile4j_of<A>());
              auto walk = [&](auto u_tag) {
              constexpr uint32_t kU = decltype(u_tag)::value;
              for (uint32_t i0 = d.lo + ct; i0 < d.hi; i0 += kU * kConsumers) {
                uint32_t tg[kU], val[kU];
                bool ok[kU];
#pragma unroll
                for (uint32_t u = 0; u < kU; ++u) {
                  const uint32_t i = i0 + u * kConsumers;
                  if constexpr (A::kMonotone) {
                    // the changed bit first: an unchanged source costs two shared
                    // loads (SrcIndexCW, its bit), not five (padding entries carry
                    // SrcIndexCW 0, a valid index, and window 0xFFFF)
                    const uint32_t l = i < d.hi ? (uint32_t)L[i] : 0u;
                    ok[u] = i < d.hi && wb_get<A>(sm, aux, wbs, l, val[u]);
                    tg[u] = 0u;
                    if (ok[u]) {
                      const uint32_t j = J[i];
                      ok[u] = j != 0xFFFFu;
                      tg[u] = (ok[u] ? drow[j] : 0u) + d.base + i;
                    }
                  } else {
                    const uint32_t j = i < d.hi ? (uint32_t)J[i] : 0xFFFFu;
                    ok[u] = j != 0xFFFFu && wb_get<A>(sm, aux, wbs, L[i], val[u]);
                    tg[u] = (ok[u] ? drow[j] : 0u) + d.base + i;
                  }
                }
#pragma unroll
                for (uint32_t u = 0; u < kU; ++u)
                  if (ok[u]) { st_u32(svq + tg[u], val[u]); ++stores; }
              }
              };
              // integer algorithms at one CTA per SM (fewer warps to hide the
              // shared-load chain of each entry): two entries per thread per step
              if ((A::kMonotone || CUSHA_S4TWO_ALL) && p.s4two) walk(std::integral_constant<uint32_t, 2>{});
              else walk(std::integral_constant<uint32_t, kS4U>{});
            } else if (any) {
              const uint16_t* L = reinterpret_cast<const uint16_t*>(ring + slot * SLOT);
              const uint32_t* M = reinterpret_cast<const uint32_t*>(ring + slot * SLOT + 2 * tile4m_of<A>());
              for (uint32_t i0 = d.lo + ct; i0 < d.hi; i0 += kS4U * kConsumers) {
                uint32_t tg[kS4U], val[kS4U];
                bool ok[kS4U];
#pragma unroll
                for (uint32_t u = 0; u < kS4U; ++u) {
                  const uint32_t i = i0 + u * kConsumers;
                  if constexpr (A::kMonotone) {  // the changed bit first (as above)
                    const uint32_t l = i < d.hi ? (uint32_t)L[i] : 0u;
                    ok[u] = i < d.hi && wb_get<A>(sm, aux, wbs, l, val[u]);
                    tg[u] = ok[u] ? M[i] : 0u;
                  } else {
                    tg[u] = i < d.hi ? M[i] : 0u;
                    ok[u] = i < d.hi && wb_get<A>(sm, aux, wbs, L[i], val[u]);
                  }
                }
#pragma unroll
                for (uint32_t u = 0; u < kS4U; ++u)
                  if (ok[u]) {
                    if (kDiag & 4) {
                      if (val[u] == 0x9e3779b9u && tg[u] == 7u) st_u32(svq + tg[u], val[u]);  // keep the loads
                    } else {
                      st_u32(svq + tg[u], val[u]);
                    }
                    ++stores;
                  }
              }
            }
            __syncwarp();
            if (lane == 0) mbar_arrive(&empty_bar[slot]);
            if (++slot == nst) { slot = 0; ph ^= 1; }
            if (d.flags & kFlagLast) {
              if (CUSHA_TIMELINE && ct == 0) tl_mark(tk, 11);
              break;
            }
          }
        }
      } else if (any) {
        // G-Shards: windows W_sj of every shard j (L151, Fig. 3c), walked a
        // batch of 32 windows per warp with one entry per lane (gs_walk)
        gs_walk(p, s, lane, cwarp, kConsumerWarps, [&](uint32_t e, uint32_t l) {
          uint32_t val;
          if (wb_get<A>(sm, aux, wbs, l, val)) { st_u32(p.sv_write + e, val); ++stores; }
        });
      }
#pragma unroll
      for (int o = 16; o; o >>= 1) stores += __shfl_xor_sync(kFull, stores, o);
      if (lane == 0 && stores) atomicAdd(&s_stores, (unsigned long long)stores);
      if (p.skip && any) __threadfence();  // release: SrcValue stores before the dirty marks below
      bar_sync(kConsumerBar, kConsumers);
      if (CUSHA_TIMELINE && ct == 0) tl_mark(tk, 6);

      if (p.skip && any) {
        // mark every shard j fed by a non-empty window W_sj (own partition; the
        // refresh marks the others) and, where local state reads the vertex's
        // own value (HS), shard s itself
        const uint32_t* w0 = p.win + (size_t)s * p.S;
        const uint32_t* w1 = w0 + p.S;
        for (uint32_t j = ct; j < p.S; j += kConsumers)
          if (__ldg(w1 + j) > __ldg(w0 + j)) {
            if (p.G == 1) {
              p.dirty[j] = 1u;
            } else {  // shard j of partition q: its flag lives with q (over NVLink on another GPU)
              const uint32_t q = p.owner[j];
              st_u32(p.dirty_peer[q] + (j - p.bounds[q]), 1u);
            }
          }
        if (A::kId == kHS && ct == 0) p.dirty[s] = 1u;
        if (p.multi) bar_sync(kConsumerBar, kConsumers);  // the marks precede the ticket's completion
      }

      // ---- per-shard bookkeeping: convergence flag (line 26), predictor, trace
      if (ct == 0) {
        if (kBk) {
          if (CUSHA_EARLY_SEQ == 1 && p.multi) {
            // the shard's next pass may start now: every consumer's stores of this
            // ticket precede this fence (barrier above; the fence is cumulative).
            // The trace / done bookkeeping follows in the bookkeeper warp; the
            // convergence argument needs only the writes complete (kernels.cu top)
            __threadfence();
            st_vol(&p.shard_seq[s], it + 1);
          }
          // hand the ticket to the bookkeeper warp (every consumer's stores precede
          // this through the barrier above; the bookkeeper's fence is cumulative)
          const uint32_t b = ntk & 1u;
          mbar_wait(&bk_empty[b], ((ntk >> 1) & 1u) ^ 1u);
          bk[b] = BkRec{s, it, (uint32_t)any, s_upd, s_stores};
          mbar_arrive(&bk_full[b]);
          ++ntk;
        } else {
          ticket_bookkeeping(p, s, it, any != 0, s_upd, s_stores, Sloc);
          if (CUSHA_TIMELINE) tl_mark(tk, 7);
        }
      }
    }
    if (kBk && ct == 0) {  // no more tickets: release the bookkeeper
      const uint32_t b = ntk & 1u;
      mbar_wait(&bk_empty[b], ((ntk >> 1) & 1u) ^ 1u);
      bk[b].s = 0xFFFFFFFFu;
      mbar_arrive(&bk_full[b]);
    }
  } else {
    // bookkeeper warp (kBk): the end-of-ticket bookkeeping, in ticket order
    if (lane == 0) {
      for (uint32_t n = 0;; ++n) {
        const uint32_t b = n & 1u;
        mbar_wait(&bk_full[b], (n >> 1) & 1u);
        const BkRec r = bk[b];
        if (r.s == 0xFFFFFFFFu) break;
        if (CUSHA_EARLY_SEQ == 2 && p.multi) {
          // release the shard's next pass first (the consumers' stores precede the
          // hand-over: barrier, then the mbarrier; this fence is cumulative), so
          // the fence's latency is off the consumers' path
          __threadfence();
          st_vol(&p.shard_seq[r.s], r.it + 1);
        }
        ticket_bookkeeping(p, r.s, r.it, r.any != 0, r.upd, r.stores, Sloc);
        if (CUSHA_TIMELINE) tl_mark(r.it * Sloc + r.s, 7);
        mbar_arrive(&bk_empty[b]);
      }
    }
  }
  __syncthreads();
  if (tid == 0) {  // every mbarrier is done with: invalidate before the shared memory is reused (PTX)
    for (uint32_t i = 0; i < nst; ++i) {
      mbar_inval(&full_bar[i]);
      mbar_inval(&empty_bar[i]);
    }
    mbar_inval(&decide_bar);
    for (uint32_t i = 0; i < 2; ++i) {
      mbar_inval(&bk_full[i]);
      mbar_inval(&bk_empty[i]);
    }
  }
  if (p.multi) return;  // overlapped passes: the last ticket of a pass closed it (ticket_done)

  // ---- iteration close (L189): the last CTA to finish decides whether another pass follows
  if (tid == 0) {
    if (p.G > 1) __threadfence_system();  // stage-4 stores into other GPUs' SrcValue / dirty before the arrival
    else __threadfence();
    const uint32_t t = atomicAdd(&p.ctl->ctas_done, 1u);
    if (t == gridDim.x - 1) {
      __threadfence();
      const uint32_t changed = *reinterpret_cast<volatile uint32_t*>(&p.ctl->changed);
      p.ctl->iter = it0 + 1;
      p.ctl->changed = 0;
      p.ctl->ctas_done = 0;
      p.ctl->next_shard = 0;
      // with G partitions the global answer is the OR over partitions (close_parts)
      if (p.G == 1) p.ctl->converged = changed ? 0u : 1u;
      else p.ctl->lchanged = changed;
      __threadfence();
    }
  }
}

// -------------------------------------------- global convergence (row e)
// After every partition's pass (and, with one process per GPU, the NCCL
// all-reduce of the partitions' lchanged words into gchanged): the run has
// converged when no partition committed an update in that pass (L189).  The
// pass is BSP across partitions - the all-reduce (or, simulated, the stream
// order) separates consecutive passes - so a pass in which nothing committed
// anywhere read a state no stage 4 changed during it: the fixed point.
//   sim = 1: ctls[0..G) are the partitions of this process; gchanged = OR lchanged.
//   sim = 0: ctls[0] is this rank's, gchanged already holds the all-reduce.
__global__ void close_parts(Ctl* const* ctls, uint32_t G, int sim) {
  if (threadIdx.x != 0) return;
  uint32_t any = 0;
  if (sim)
    for (uint32_t q = 0; q < G; ++q) any |= *reinterpret_cast<volatile uint32_t*>(&ctls[q]->lchanged);
  else
    any = *reinterpret_cast<volatile uint32_t*>(&ctls[0]->gchanged);
  for (uint32_t q = 0; q < (sim ? G : 1u); ++q) {
    Ctl* c = ctls[q];
    if (!c->converged && c->iter >= 1 && !any) c->converged = 1u;
  }
}

// ------------------------------------------------------------ init kernels
// VertexValues <- Table-3 start state (L327) or the user's initial values for
// the partition's vertices; every shard predicted active for the first pass.
template <class A>
__global__ void init_vertex_values(const KParams p, const void* user, uint32_t v0, uint32_t nvl) {
  using V_t = typename A::Value;
  V_t* vv = reinterpret_cast<V_t*>(p.vv);
  const V_t* u = reinterpret_cast<const V_t*>(user);
  for (size_t v = blockIdx.x * (size_t)blockDim.x + threadIdx.x; v < nvl; v += (size_t)gridDim.x * blockDim.x)
    vv[v] = u ? u[v] : A::start((uint32_t)(v0 + v), p.source);
  for (size_t s = blockIdx.x * (size_t)blockDim.x + threadIdx.x; s < p.Sl; s += (size_t)gridDim.x * blockDim.x) {
    p.active[s] = 1;
    if (p.dirty) p.dirty[s] = 1u;  // every shard runs the first pass
    p.shard_seq[s] = 0;
  }
}

// SrcValue[e] <- VertexValues[SrcIndex[e]] for every entry (R20: a full
// write-back at t = 0), one CTA per own source shard i.  Every source of shard
// i's windows lies in shard i, so the CTA first stages the write-back values of
// its |N| vertices in shared memory (coalesced) and then streams its windows
// (G-Shards) or CW_i (CW) against them, as stage 4 of a pass does - into every
// partition's SrcValue when the graph is partitioned.
template <class A>
__device__ __forceinline__ void stage_wb_values(const KParams& p, uint32_t i, uint32_t* wb) {
  using V_t = typename A::Value;
  const V_t* vv = reinterpret_cast<const V_t*>(p.vv);
  const uint32_t off = i * p.N, nv = min(p.N, p.V - (p.s0 + i) * p.N);
  for (uint32_t v = threadIdx.x; v < nv; v += blockDim.x)
    wb[v] = A::wb_value(vv[off + v], A::kOutDeg ? __ldg(p.outdeg + off + v) : 0u);
  __syncthreads();
}
template <class A>
__global__ void __launch_bounds__(512) init_srcvalue_gs(const KParams p) {
  extern __shared__ uint32_t wb[];
  const uint32_t i = blockIdx.x, lane = threadIdx.x & 31u, warp = threadIdx.x >> 5;
  stage_wb_values<A>(p, i, wb);
  gs_walk(p, i, lane, warp, blockDim.x / 32, [&](uint32_t e, uint32_t l) { p.srcvalue[e] = wb[l]; });
}
template <class A>
__global__ void __launch_bounds__(512) init_srcvalue_cw(const KParams p) {
  extern __shared__ uint32_t wb[];
  const uint32_t i = blockIdx.x;
  stage_wb_values<A>(p, i, wb);
  for (uint32_t q = 0; q < p.G; ++q) {
    uint32_t a, b;
    if (p.G > 1) {
      a = p.cwp[(size_t)i * (p.G + 1) + q];
      b = p.cwp[(size_t)i * (p.G + 1) + q + 1];
    } else {
      a = p.cw_off[i];
      b = a + p.cw_cnt[i];
    }
    uint32_t* const svq = p.G > 1 ? p.sv_peer[q] : p.srcvalue;
    for (uint32_t k = a + threadIdx.x; k < b; k += blockDim.x) {
      uint32_t m;
      if (p.mapper) m = __ldg(topo_at(p.mapper, p.mapper_h, p.splitQ, k));
      else m = __ldg(p.cw_delta + (size_t)i * p.S + __ldg(topo_at(p.cw_win, p.cw_win_h, p.splitQ, k))) + k;
      svq[m] = wb[__ldg(topo_at(p.cw_src, p.cw_src_h, p.splitQ, k))];
    }
  }
}

// One partition (G = 1): SrcValue[Mapper[k]] = wb_value(VertexValues[SrcIndexCW[k]])
// over every CW entry k (R20), one block per chunk of kInitChunk entries of one
// CW_i (chunks[b] = (i, first position)), 8 entries per thread with every
// load issued before the stores: the entries are independent, so the stream
// runs at bandwidth instead of one dependent chain per thread and shard.
template <class A>
// from_start: VertexValues hold A::start (no user initial values), so the
// value is computed from the vertex id instead of loaded (PR: Rank 1, CC: the id)
__global__ void __launch_bounds__(256, 8) init_srcvalue_cw_flat(const KParams p, const uint2* chunks, int from_start) {
  using V_t = typename A::Value;
  constexpr uint32_t kU = kInitChunk / 256;
  const uint2 c = chunks[blockIdx.x];
  const uint32_t i = c.x, e = min(c.y + kInitChunk, p.cw_off[i] + p.cw_cnt[i]);
  const V_t* vv = reinterpret_cast<const V_t*>(p.vv) + (size_t)i * p.N;
  const uint32_t* od = p.outdeg + (size_t)i * p.N;
  const uint32_t* drow = p.cw_delta + (size_t)i * p.S;
  uint32_t l[kU], m[kU];
#pragma unroll
  for (uint32_t u = 0; u < kU; ++u) {
    const uint32_t k = c.y + u * 256 + threadIdx.x;
    l[u] = 0;
    m[u] = 0;
    if (k < e) {
      l[u] = __ldg(topo_at(p.cw_src, p.cw_src_h, p.splitQ, k));
      m[u] = p.mapper ? __ldg(topo_at(p.mapper, p.mapper_h, p.splitQ, k)) : __ldg(topo_at(p.cw_win, p.cw_win_h, p.splitQ, k));
    }
  }
  uint32_t val[kU];
#pragma unroll
  for (uint32_t u = 0; u < kU; ++u) {
    const uint32_t k = c.y + u * 256 + threadIdx.x;
    if (k < e) {
      if (!p.mapper) m[u] = __ldg(drow + m[u]) + k;
      const V_t x = from_start ? A::start((p.s0 + i) * p.N + l[u], p.source) : vv[l[u]];
      val[u] = A::wb_value(x, A::kOutDeg ? __ldg(od + l[u]) : 0u);
    }
  }
#pragma unroll
  for (uint32_t u = 0; u < kU; ++u)
    if (c.y + u * 256 + threadIdx.x < e) p.srcvalue[m[u]] = val[u];
}

// Start states uniform except at the source (A::kUniformStart, one partition):
// SrcValue at t = 0 is wb_value(start(v)) = U for every source v but the BFS /
// SSSP / SSWP source, so the R20 write-back is a fill of every entry (filler
// entries included: they reduce into the trash slot) followed by a patch of the
// source's out-edges - a write-only stream instead of a gather per entry.
__global__ void fill_u32(uint32_t* a, uint64_t n, uint32_t v) {
  const uint64_t n4 = n / 4;
  uint4* a4 = reinterpret_cast<uint4*>(a);  // SrcValue is 256-B aligned (pool allocation)
  const uint4 q = make_uint4(v, v, v, v);
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n4; i += (uint64_t)gridDim.x * blockDim.x)
    a4[i] = q;
  for (uint64_t i = n4 * 4 + blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x)
    a[i] = v;
}
// the source's out-edges: its shard i's CW_i entries with SrcIndexCW == the
// source's local index (CW), or its windows W_ij (G-Shards)
template <class A>
__global__ void patch_source_cw(const KParams p, uint32_t i, uint32_t lsrc, uint32_t val) {
  const uint32_t a = p.cw_off[i], b = a + p.cw_cnt[i];
  const uint32_t* drow = p.cw_delta + (size_t)i * p.S;
  for (uint32_t k = a + blockIdx.x * blockDim.x + threadIdx.x; k < b; k += gridDim.x * blockDim.x)
    if (__ldg(topo_at(p.cw_src, p.cw_src_h, p.splitQ, k)) == lsrc) {
      const uint32_t m = p.mapper ? __ldg(topo_at(p.mapper, p.mapper_h, p.splitQ, k))
                                  : __ldg(drow + __ldg(topo_at(p.cw_win, p.cw_win_h, p.splitQ, k))) + k;
      p.srcvalue[m] = val;
    }
}
__global__ void __launch_bounds__(512) patch_source_gs(const KParams p, uint32_t i, uint32_t lsrc, uint32_t val) {
  const uint32_t lane = threadIdx.x & 31u, warp = threadIdx.x >> 5;
  gs_walk(p, i, lane, warp, blockDim.x / 32, [&](uint32_t e, uint32_t l) {
    if (l == lsrc) p.srcvalue[e] = val;
  });
}

__global__ void reset_ctl(Ctl* ctl, uint32_t max_iters) {
  ctl->iter = 0;
  ctl->changed = 0;
  ctl->ctas_done = 0;
  ctl->max_iters = max_iters;
  ctl->converged = 0;
  ctl->next_shard = 0;
  ctl->lchanged = 0;
  ctl->gchanged = 0;
  ctl->ticket = 0;
  ctl->stop = 0;
  ctl->conv_iter = 0xFFFFFFFFu;
}

// -------------------------------------------------------------- dispatch
size_t PassKernel::smem_bytes(uint32_t N, uint32_t delta_row) const {
  size_t w = (size_t)words * (N + 1);  // (float write-back values overlay the first sum word)
  if (monotone) w += (N + 31) / 32;
  return ring_bytes + 4 * (w + delta_row);
}

template <class A, int R>
static PassKernel make_pk() {
  PassKernel k;
  k.func = reinterpret_cast<const void*>(&shard_pass<A, R>);
  k.words = A::kWords;
  k.wb_array = !A::kMonotone;
  k.monotone = A::kMonotone;
  k.ring_bytes = kStages * slot_bytes<A>();
  k.slot_bytes = slot_bytes<A>();
  k.max_stages = kMaxStages;
  k.threads = kPassThreads;
  k.persistent = kPersistent;
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


bool kernels_rle() { return kRle; }

// diagnostic timeline builds only: copy the stamps out (tools/timeline.py)
int timeline_copy(void* out, size_t bytes) {
#if CUSHA_TIMELINE
  const size_t n = bytes < sizeof(g_timeline) ? bytes : sizeof(g_timeline);
  return cudaMemcpyFromSymbol(out, g_timeline, n) == cudaSuccess ? (int)(n / (4 * kTlSlots)) : -1;
#else
  (void)out; (void)bytes;
  return -1;
#endif
}

size_t value_bytes(int alg) { return (alg == kHS || alg == kCS) ? 8 : 4; }
bool alg_needs_edge_values(int alg) { return alg == kSSSP || alg == kSSWP || alg == kNN || alg == kHS || alg == kCS; }
bool alg_needs_init(int alg) { return alg == kNN || alg == kHS || alg == kCS; }

KParams make_params(const Graph& g, uint32_t source) {
  KParams p{};
  p.V = g.V; p.N = g.N; p.S = g.S; p.source = source;
  p.s0 = g.s0; p.Sl = g.Sl;
  p.shard_off = g.d_shard_off; p.shard_cnt = g.d_shard_cnt; p.dest = g.d_dest; p.ev = g.d_ev; p.srcvalue = g.d_srcvalue;
  p.sv_write = g.d_srcvalue;
  p.sv_peer = g.d_sv_peer;
  p.srcloc = g.d_srcloc; p.win = g.d_win; p.cw_off = g.d_cw_off; p.cw_cnt = g.d_cw_cnt; p.active = g.d_active;
  p.cw_src = g.d_cw_src; p.mapper = g.d_mapper; p.vv = g.d_vv; p.outdeg = g.d_outdeg;
  p.cw_win = g.d_cw_win; p.cw_delta = g.d_cw_delta; p.cw_win_h = g.h_cw_win;
  p.ctl = g.d_ctl; p.trace = g.d_trace; p.trace_cap = g.trace_cap;
  p.G = g.G;
  p.bounds = g.d_bounds; p.owner = g.d_owner; p.cwp = g.d_cwp; p.dirty_peer = g.d_dirty_peer;
  p.run_k = g.d_run_k; p.run_t = g.d_run_t; p.run_unit = g.d_run_unit; p.run_bits = g.d_run_bits; p.run_d = g.d_run_d;
  p.R = g.R;
  p.skip = g.skip_clean ? 1 : 0; p.dirty = g.d_dirty;
  p.splitP = (uint32_t)g.splitP; p.splitQ = (uint32_t)g.splitQ;
  p.dest_h = g.h_dest; p.ev_h = g.h_ev; p.srcloc_h = g.h_srcloc; p.cw_src_h = g.h_cw_src; p.mapper_h = g.h_mapper;
  p.multi = 0; p.shard_seq = g.d_shard_seq;
  p.order = nullptr;
  p.window = 2;
  p.mapj = 0;
  p.stash = 0;
  p.ahead = 0;
  p.nst = kStages;
  p.s4two = 0;
  return p;
}

// cudaFuncSetAttribute once per (kernel, device, size): the per-run launch
// path then makes no attribute calls
static cudaError_t smem_attr(const void* fn, size_t bytes) {
  static std::mutex mu;
  static std::map<std::pair<const void*, int>, size_t> done;
  int dev = 0;
  cudaGetDevice(&dev);
  std::lock_guard<std::mutex> lock(mu);
  size_t& have = done[{fn, dev}];
  if (have >= bytes) return cudaSuccess;
  const cudaError_t e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)bytes);
  if (e == cudaSuccess) have = bytes;
  return e;
}

template <class A>
static cudaError_t launch_init_t(const Graph& g, uint32_t source, cudaStream_t s) {
  KParams p = make_params(g, source);
  const uint32_t vb = (uint32_t)((g.nvl + 255) / 256);
  init_vertex_values<A><<<vb < 148 * 16 ? (vb ? vb : 1) : 148 * 16, 256, 0, s>>>(p, g.d_init[A::kId], g.v0, g.nvl);
  if (g.Sl && A::kUniformStart && g.G == 1 && !g.d_init[A::kId] && source < g.V) {
    // host copies of start(): U for every vertex but the source, the source's own
    uint32_t U = 0, Vs = 0;
    if (A::kId == kSSWP) { U = 0u; Vs = kInf; } else { U = kInf; Vs = 0u; }
    const uint64_t n = g.P + 1;
    const uint64_t blocks = std::min<uint64_t>((n / 4 + 255) / 256 + 1, 148ull * 16);
    fill_u32<<<(uint32_t)blocks, 256, 0, s>>>(g.d_srcvalue, n, U);
    const uint32_t i = source / g.N, lsrc = source - i * g.N;
    if (g.repr == CUSHA_REPR_CW) patch_source_cw<A><<<148, 256, 0, s>>>(p, i, lsrc, Vs);
    else patch_source_gs<<<1, 512, 0, s>>>(p, i, lsrc, Vs);
    return cudaGetLastError();
  }
  if (g.Sl) {
    const size_t sm = 4ull * g.N;  // the shard's write-back values (|N| <= 65534: at most 256 KB)
    const void* fn = g.repr == CUSHA_REPR_CW ? (const void*)&init_srcvalue_cw<A> : (const void*)&init_srcvalue_gs<A>;
    cudaError_t e = smem_attr(fn, sm);
    if (e != cudaSuccess) return e;  // |N| beyond the shared-memory limit cannot run the pass either
    if (g.repr == CUSHA_REPR_CW && g.G == 1 && g.d_init_chunks) {
      if (g.init_nchunks)
        init_srcvalue_cw_flat<A><<<g.init_nchunks, 256, 0, s>>>(p, g.d_init_chunks, g.d_init[A::kId] ? 0 : 1);
    } else if (g.repr == CUSHA_REPR_CW) {
      init_srcvalue_cw<A><<<g.Sl, 512, sm, s>>>(p);
    } else {
      init_srcvalue_gs<A><<<g.Sl, 512, sm, s>>>(p);
    }
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

// ------------------------------------ barrier between ranks (row e, one process per GPU)
// After a pass: every rank stores its "committed an update" word into every
// rank's block, then counts itself in; it waits until all G ranks arrived, and
// the run has converged when no rank committed (L189).  The same G words
// reach every rank, so all take the same decision.  A rank re-uses a slot two
// rounds later only after every rank passed the round in between, which needs
// this rank's arrival there - issued after the reset below.  Bounded: after
// timeout_ms the rank flags err and stops its run instead of spinning forever.
__global__ void peer_barrier(PeerSync* const* peers, uint32_t G, uint32_t rank, Ctl* ctl, uint32_t timeout_ms,
                             int decide) {
  if (threadIdx.x != 0) return;
  __threadfence_system();  // this rank's pass (its stage-4 stores to the peers) before the arrival
  PeerSync* me = peers[rank];
  const uint32_t r = ld_vol(&me->round), par = r & 1u;
  const uint32_t v = decide ? ld_vol(&ctl->lchanged) : 0u;
  for (uint32_t q = 0; q < G; ++q) st_vol(&peers[q]->changed[par][rank], v);
  __threadfence_system();
  for (uint32_t q = 0; q < G; ++q) atomicAdd_system(&peers[q]->arrive[par], 1u);
  uint64_t t0, t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
  while (ld_vol(&me->arrive[par]) < G) {
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    if (t - t0 > (uint64_t)timeout_ms * 1000000ull) {
      me->err = 1u;
      ctl->converged = 1u;  // stop this rank's run; the host reports the timeout
      break;
    }
    __nanosleep(256);
  }
  __threadfence_system();
  uint32_t any = 0;
  for (uint32_t q = 0; q < G; ++q) any |= ld_vol(&me->changed[par][q]);
  if (decide && !ctl->converged && ctl->iter >= 1 && !any) ctl->converged = 1u;
  st_vol(&me->arrive[par], 0u);
  st_vol(&me->round, r + 1);
  __threadfence_system();
}

cudaError_t launch_peer_barrier(const Graph& g, int decide, uint32_t timeout_ms, cudaStream_t s) {
  peer_barrier<<<1, 32, 0, s>>>(g.d_sync_peer, g.G, g.part, g.d_ctl, timeout_ms, decide);
  return cudaGetLastError();
}

cudaError_t launch_close_parts(Ctl* const* ctls, uint32_t G, cudaStream_t s) {
  // ctls: device array; G > 0: all partitions of this process (simulation); G == 0: one rank after its all-reduce
  close_parts<<<1, 32, 0, s>>>(ctls, G ? G : 1u, G ? 1 : 0);
  return cudaGetLastError();
}

cudaError_t launch_reset_ctl(Ctl* ctl, uint32_t max_iters, cudaStream_t s) {
  reset_ctl<<<1, 1, 0, s>>>(ctl, max_iters);
  return cudaGetLastError();
}

}  // namespace cusha
