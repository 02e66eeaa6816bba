// lcf_pipe.cuh — sm_100a pipeline primitives: mbarriers, 1-D TMA bulk copies
// (cp.async.bulk, SASS UBLKCP), proxy fences, named barriers, clamped shifts.
#pragma once
#include <stdint.h>

namespace lcf {

__device__ __forceinline__ uint32_t smem_addr(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

// ---- mbarrier ----------------------------------------------------------------
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_addr(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
  asm volatile("mbarrier.arrive.release.cta.shared::cta.b64 _, [%0];" ::"r"(smem_addr(bar)) : "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.release.cta.shared::cta.b64 _, [%0], %1;" ::"r"(smem_addr(bar)),
               "r"(bytes)
               : "memory");
}
__device__ __forceinline__ bool mbar_try_wait(uint64_t* bar, uint32_t parity) {
  uint32_t ok;
  asm volatile(
      "{\n .reg .pred p;\n mbarrier.try_wait.parity.acquire.cta.shared::cta.b64 p, [%1], %2;\n selp.u32 %0, 1, 0, p;\n}"
      : "=r"(ok)
      : "r"(smem_addr(bar)), "r"(parity)
      : "memory");
  return ok != 0;
}
#ifndef LCF_MBAR_HINT
#define LCF_MBAR_HINT 0
#endif
// try_wait with a suspend-time hint (ns): the waiting warp is descheduled until
// the phase completes or the hint expires, instead of spinning on issue slots.
__device__ __forceinline__ bool mbar_try_wait_hint(uint64_t* bar, uint32_t parity, uint32_t ns) {
  uint32_t ok;
  asm volatile(
      "{\n .reg .pred p;\n mbarrier.try_wait.parity.acquire.cta.shared::cta.b64 p, [%1], %2, %3;\n"
      " selp.u32 %0, 1, 0, p;\n}"
      : "=r"(ok)
      : "r"(smem_addr(bar)), "r"(parity), "r"(ns)
      : "memory");
  return ok != 0;
}
#ifndef LCF_MBAR_SLEEP
#define LCF_MBAR_SLEEP 0
#endif
// A waiting warp backs off with __nanosleep (32 ns doubling up to
// LCF_MBAR_SLEEP ns; 0 = spin): a spinning loader or storer warp otherwise
// issues try_wait loops on the same scheduler as the compute warps (ncu on
// SPratio/NYX: 28 % of the encoder's warp instructions were wait loops).
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
#if LCF_MBAR_HINT
  while (!mbar_try_wait_hint(bar, parity, LCF_MBAR_HINT)) {
  }
#elif LCF_MBAR_SLEEP
  uint32_t ns = 32;
  while (!mbar_try_wait(bar, parity)) {
    __nanosleep(ns);
    ns = ns < LCF_MBAR_SLEEP ? 2 * ns : ns;
  }
#else
  while (!mbar_try_wait(bar, parity)) {
  }
#endif
}

// ---- TMA bulk copies (non-tensor, 16-byte granules) ---------------------------
__device__ __forceinline__ void tma_load_1d(void* smem_dst, const void* gmem_src, uint32_t bytes, uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
          smem_addr(smem_dst)),
      "l"(gmem_src), "r"(bytes), "r"(smem_addr(bar))
      : "memory");
}
// 2-D tensor load of the box at tensor coordinates (c0, c1) into smem_dst (laid
// out as the tensor map's swizzle mode prescribes), completing on `bar`
__device__ __forceinline__ void tma_load_2d(void* smem_dst, const void* tmap, int32_t c0, int32_t c1, uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];" ::"r"(
          smem_addr(smem_dst)),
      "l"(tmap), "r"(c0), "r"(c1), "r"(smem_addr(bar))
      : "memory");
}
__device__ __forceinline__ void tma_store_1d(void* gmem_dst, const void* smem_src, uint32_t bytes) {
  asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(gmem_dst),
               "r"(smem_addr(smem_src)), "r"(bytes)
               : "memory");
}
// 2-D tensor store of the box at smem_src (laid out as the tensor map's
// swizzle mode prescribes) to tensor coordinates (c0, c1)
__device__ __forceinline__ void tma_store_2d(const void* tmap, const void* smem_src, int32_t c0, int32_t c1) {
  asm volatile("cp.async.bulk.tensor.2d.global.shared::cta.bulk_group [%0, {%1, %2}], [%3];" ::"l"(tmap), "r"(c0),
               "r"(c1), "r"(smem_addr(smem_src))
               : "memory");
}
__device__ __forceinline__ void tma_store_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
__device__ __forceinline__ void tma_store_wait_read0() {
  asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
}
__device__ __forceinline__ void tma_store_wait_read1() {
  asm volatile("cp.async.bulk.wait_group.read 1;" ::: "memory");
}
__device__ __forceinline__ void tma_store_wait_all0() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }
// generic-proxy shared-memory writes → visible to the async (TMA) proxy
__device__ __forceinline__ void fence_proxy_async_smem() {
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}

// The warp's index, broadcast from lane 0: ptxas then knows that a branch on it
// (the warp-role dispatch of the persistent kernels) is warp-uniform, and
// compiles the warp-synchronous code behind it (shuffles, votes, redux) without
// WARPSYNC.COLLECTIVE / ENDCOLLECTIVE convergence wrappers. Requires the whole
// warp to be active at the call (kernel entry).
__device__ __forceinline__ uint32_t warp_index_uniform() {
  return __shfl_sync(0xFFFFFFFFu, threadIdx.x >> 5, 0);
}

// A value the caller knows to be warp-uniform (read from shared memory by
// every lane, or the result of a CTA-wide barrier reduction), broadcast from
// lane 0 so that ptxas can prove it uniform too (same reason as above).
__device__ __forceinline__ uint32_t warp_uniform(uint32_t v) { return __shfl_sync(0xFFFFFFFFu, v, 0); }
__device__ __forceinline__ uint64_t warp_uniform(uint64_t v) { return __shfl_sync(0xFFFFFFFFu, v, 0); }

// ---- named barriers (id 0 is __syncthreads) ------------------------------------
__device__ __forceinline__ void named_bar_sync(uint32_t id, uint32_t nthreads) {
  asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(nthreads) : "memory");
}

// ---- shifts with PTX clamping semantics (shift ≥ 32 → 0 / whole word) ----------
__device__ __forceinline__ uint32_t shl_c(uint32_t x, uint32_t s) {  // x << s, 0 if s ≥ 32
  uint32_t r;
  asm("shl.b32 %0, %1, %2;" : "=r"(r) : "r"(x), "r"(s));
  return r;
}
__device__ __forceinline__ uint32_t shr_c(uint32_t x, uint32_t s) {  // x >> s, 0 if s ≥ 32
  uint32_t r;
  asm("shr.b32 %0, %1, %2;" : "=r"(r) : "r"(x), "r"(s));
  return r;
}

}  // namespace lcf
