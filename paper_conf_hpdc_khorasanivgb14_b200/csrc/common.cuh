// common.cuh — device helpers shared by the CuSha kernels (product path only).
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace cusha {

constexpr uint32_t kInf = 0xFFFFFFFFu;   // DESIGN.md R1 (Table 3 "INF")
constexpr uint32_t kPad = 8;             // entries per vector chunk: shards / CW_i padded to multiples of 8

// ---------------------------------------------------------------- loads
// SrcValue is written by other CTAs' stage 4 during the same launch (the
// asynchronous model of L45), so it is read with ld.global.cg (L2, never a
// possibly stale L1 line and never the non-coherent path).  Topology arrays
// are read-only for the whole run: non-coherent, no L1 allocation.
__device__ __forceinline__ uint4 ld_cg_v4(const void* p) {
  uint4 r;
  asm volatile("ld.global.cg.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p));
  return r;
}
__device__ __forceinline__ uint4 ld_stream_v4(const void* p) {
  uint4 r;
  asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
               : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w)
               : "l"(p));
  return r;
}
__device__ __forceinline__ uint32_t ld_ro(const uint32_t* p) { return __ldg(p); }
__device__ __forceinline__ void st_u32(uint32_t* p, uint32_t v) {
  asm volatile("st.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

// ------------------------------------------- TMA bulk copies + mbarriers
// 1-D cp.async.bulk global -> shared (TMA engine) completing on an mbarrier
// with a transaction count; the producer/consumer ring of the shard pass.
__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_inval(uint64_t* bar) {
  asm volatile("mbarrier.inval.shared::cta.b64 [%0];" ::"r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void mbar_fence_init() {
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  uint32_t done = 0;
  do {
    asm volatile(
        "{\n .reg .pred p;\n mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n selp.u32 %0, 1, 0, p;\n}\n"
        : "=r"(done)
        : "r"(smem_u32(bar)), "r"(parity)
        : "memory");
  } while (!done);
}
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                   smem_u32(dst)),
               "l"(src), "r"(bytes), "r"(smem_u32(bar))
               : "memory");
}

// Ampere-style asynchronous 4-byte global -> shared copy (LDGSTS), per thread
__device__ __forceinline__ void cp_async4(void* dst, const void* src) {
  asm volatile("cp.async.ca.shared.global [%0], [%1], 4;" ::"r"(smem_u32(dst)), "l"(src) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
__device__ __forceinline__ void cp_async_wait_all() { asm volatile("cp.async.wait_all;" ::: "memory"); }

// TMA bulk prefetch of [src, src + bytes) into L2 (no shared memory, no
// completion to wait for); the range is widened to 16-byte bounds
__device__ __forceinline__ void bulk_prefetch_l2(const void* src, uint32_t bytes) {
  const uintptr_t a = reinterpret_cast<uintptr_t>(src) & ~uintptr_t(15);
  const uint32_t n = (uint32_t)(((reinterpret_cast<uintptr_t>(src) + bytes + 15) & ~uintptr_t(15)) - a);
  if (n) asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(a), "r"(n) : "memory");
}

// L2 policy for streams read once per pass (topology arrays): evict first, so
// that SrcValue lines written by stage 4 stay in L2 until stage 2 reads them
__device__ __forceinline__ uint64_t l2_evict_first_policy() {
  uint64_t pol;
  asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
  return pol;
}
__device__ __forceinline__ void bulk_g2s_hint(void* dst, const void* src, uint32_t bytes, uint64_t* bar,
                                              uint64_t pol) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;" ::
          "r"(smem_u32(dst)),
      "l"(src), "r"(bytes), "r"(smem_u32(bar)), "l"(pol)
      : "memory");
}

// named barrier over `count` threads; returns the OR of pred over them
__device__ __forceinline__ int bar_sync_or(uint32_t id, uint32_t count, int pred) {
  int r;
  asm volatile(
      "{\n .reg .pred p, q;\n setp.ne.s32 p, %1, 0;\n bar.red.or.pred q, %2, %3, p;\n selp.s32 %0, 1, 0, q;\n}\n"
      : "=r"(r)
      : "r"(pred), "r"(id), "r"(count)
      : "memory");
  return r;
}
__device__ __forceinline__ void bar_sync(uint32_t id, uint32_t count) {
  asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(count) : "memory");
}

// --------------------------------------------------- 64-bit fixed point
// Float sums of Table 3 (PR, NN, HS, CS) are accumulated in shared memory as
// 64-bit two's-complement fixed point with 32 fraction bits, using native
// 32-bit ATOMS.ADD on a lo word and carrying into a hi word (f32 shared
// atomicAdd is a CAS loop on sm_100a; u32 add is native).  Integer addition
// is associative, so the sum is independent of the atomic order
// (R11: frozen inputs give frozen sums, so PR terminates).
// x * 2^32 (exact power-of-two scaling) truncated toward zero to a 64-bit
// two's-complement integer (F2I.S64).  Exact for |x| < 2^31; larger
// magnitudes saturate (never reached: DESIGN.md R11).  (An integer-shift
// version was measured slower on B200: tools/tune.)
__device__ __forceinline__ uint64_t f2fix(float x) {
  return (uint64_t)__float2ll_rz(x * 4294967296.0f);
}
__device__ __forceinline__ float fix2f(uint32_t lo, uint32_t hi) {
  long long v = (long long)(((uint64_t)hi << 32) | lo);
  return ldexpf(__ll2float_rn(v), -32);
}
__device__ __forceinline__ void fix_add(uint32_t* lo, uint32_t* hi, uint64_t F) {
  uint32_t l = (uint32_t)F, h = (uint32_t)(F >> 32);
  uint32_t old = atomicAdd(lo, l);
  h += (old + l < old) ? 1u : 0u;  // carry out of the low word
  if (h) atomicAdd(hi, h);
}

}  // namespace cusha
