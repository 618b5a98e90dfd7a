// ptx.cuh -- PTX wrappers shared by the TMA-staged kernels (kernels_stream.cu,
// kernels_sweep.cu): mbarriers, bulk tensor copies, release/acquire status
// words, shared-memory loads by 32-bit address, the per-CTA timeline.
#pragma once

#include <cuda.h>

#include <cstdint>

#include "magus_internal.h"

#ifndef MAGUS_LOOKBACK_SLEEP
#define MAGUS_LOOKBACK_SLEEP 32  // ns between polls of a predecessor's segment status
#endif

namespace magus {
namespace {

__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return (uint32_t)__cvta_generic_to_shared(p);
}
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)),
               "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}
// try_wait with a suspend-time hint: a waiting warp is parked by the hardware
// instead of re-issuing the probe (the producer otherwise burns ~20 % of the
// SM's issue slots spinning on the empty barriers).
__device__ __forceinline__ void mbar_wait_s(uint32_t bar, uint32_t parity) {
  asm volatile(
      "{\n"
      ".reg .pred p;\n"
      "WAIT_%=:\n"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1, %2;\n"
      "@!p bra WAIT_%=;\n"
      "}\n" ::"r"(bar),
      "r"(parity), "r"(0x989680u)
      : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  mbar_wait_s(smem_u32(bar), parity);
}
#ifndef MAGUS_FULLWAIT_SLEEP
#define MAGUS_FULLWAIT_SLEEP 0  // ns slept between the consumers' polls of a stage (0: suspend hint only)
#endif
// the consumers' wait for a stage: with MAGUS_FULLWAIT_SLEEP > 0 a warp that
// finds the stage not yet landed sleeps between polls instead of re-issuing
// the probe (the polls of 16 waiting warps otherwise take issue slots from
// the warps doing the work)
__device__ __forceinline__ void mbar_wait_full(uint32_t bar, uint32_t parity) {
  if constexpr (MAGUS_FULLWAIT_SLEEP > 0) {
    uint32_t ok;
    asm volatile("{\n.reg .pred p;\nmbarrier.test_wait.parity.shared::cta.b64 p, [%1], %2;\nselp.u32 %0, 1, 0, p;\n}"
                 : "=r"(ok) : "r"(bar), "r"(parity) : "memory");
    while (!ok) {
      __nanosleep(MAGUS_FULLWAIT_SLEEP);
      asm volatile("{\n.reg .pred p;\nmbarrier.test_wait.parity.shared::cta.b64 p, [%1], %2;\nselp.u32 %0, 1, 0, p;\n}"
                   : "=r"(ok) : "r"(bar), "r"(parity) : "memory");
    }
  } else {
    mbar_wait_s(bar, parity);
  }
}
__device__ __forceinline__ void mbar_arrive_s(uint32_t bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(bar) : "memory");
}
// shared-window loads by 32-bit address (the generic->shared conversion of a
// pointer costs an S2R + LEA each time the compiler rematerialises it)
__device__ __forceinline__ float lds_f32(uint32_t a) {
  float v;
  asm volatile("ld.shared.f32 %0, [%1];" : "=f"(v) : "r"(a));
  return v;
}
__device__ __forceinline__ unsigned long long lds_u64(uint32_t a) {
  unsigned long long v;
  asm volatile("ld.shared.u64 %0, [%1];" : "=l"(v) : "r"(a));
  return v;
}
__device__ __forceinline__ uint4 lds_v4(uint32_t a) {
  uint4 v;
  asm volatile("ld.shared.v4.u32 {%0, %1, %2, %3}, [%4];"
               : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "r"(a));
  return v;
}
__device__ __forceinline__ void tma_load_2d(void* dst, const CUtensorMap* map, uint64_t* bar,
                                            int32_t c0, int32_t c1) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes"
      " [%0], [%1, {%3, %4}], [%2];" ::"r"(smem_u32(dst)),
      "l"(reinterpret_cast<uint64_t>(map)), "r"(smem_u32(bar)), "r"(c0), "r"(c1)
      : "memory");
}
__device__ __forceinline__ void tma_load_1d(void* dst, const CUtensorMap* map, uint64_t* bar,
                                            int32_t c0) {
  asm volatile(
      "cp.async.bulk.tensor.1d.shared::cluster.global.mbarrier::complete_tx::bytes"
      " [%0], [%1, {%3}], [%2];" ::"r"(smem_u32(dst)),
      "l"(reinterpret_cast<uint64_t>(map)), "r"(smem_u32(bar)), "r"(c0)
      : "memory");
}
__device__ __forceinline__ void st_release(uint32_t* p, uint32_t v) {
  asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ uint32_t ld_acquire(const uint32_t* p) {
  uint32_t v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ unsigned long long gtimer() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
// MAGUS_OPT_TRACE: slot i of this CTA's timeline row (the CTA index is
// re-read here so no address stays live across the scan)
__device__ __forceinline__ unsigned long long* trace_buf(const StreamWork& wk) {
  return *reinterpret_cast<unsigned long long* volatile*>(wk.ticket + kTraceSlotWords);
}
__device__ __forceinline__ void trace_put(unsigned long long* tr, int i, unsigned long long v) {
  uint32_t cta;
  asm volatile("mov.u32 %0, %%ctaid.x;" : "=r"(cta));
  tr[8ull * cta + i] = v;
}

// The warp's sum of one per-trace totals field (each lane's value < 2^32):
// counts (<= T <= 2^24 per trace, so the warp's sum < 2^29) by one
// redux.sync, the 32-bit halves of the q sums (fields 7..12) by two on
// 16-bit pieces -- exact, without five rounds of 64-bit shuffles.
__device__ __forceinline__ unsigned long long warp_sum_tot(unsigned long long v, int q) {
  const uint32_t v32 = (uint32_t)v;
  if (q >= 7 && q <= 12)
    return (unsigned long long)__reduce_add_sync(0xFFFFFFFFu, v32 & 0xFFFFu) +
           ((unsigned long long)__reduce_add_sync(0xFFFFFFFFu, v32 >> 16) << 16);
  return (unsigned long long)__reduce_add_sync(0xFFFFFFFFu, v32);
}

__device__ __forceinline__ uint32_t tail_mask(int64_t p0, int64_t T) {
  return (p0 + 32 <= T) ? ~0u : ((1u << (uint32_t)(T - p0)) - 1u);
}

}  // namespace
}  // namespace magus
