// kcommon.cuh — device helpers shared by the libarbalest kernels.
#pragma once
#include "arb_internal.h"

namespace arb {

#define FULL 0xFFFFFFFFu

__device__ __forceinline__ uint32_t lanemask_lt() {
  uint32_t m;
  asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
  return m;
}

// streaming (evict-first) loads of data read exactly once
__device__ __forceinline__ uint4 ld_stream(const uint4* p) {
  uint4 r;
  asm volatile("ld.global.cs.v4.u32 {%0,%1,%2,%3}, [%4];"
               : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p));
  return r;
}

// ---- cp.async staging -------------------------------------------------------
__device__ __forceinline__ void cp_async16(void* smem_dst, const void* gsrc) {
  const uint32_t d = (uint32_t)__cvta_generic_to_shared(smem_dst);
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(d), "l"(gsrc) : "memory");
}
__device__ __forceinline__ void cp_async8(void* smem_dst, const void* gsrc) {
  const uint32_t d = (uint32_t)__cvta_generic_to_shared(smem_dst);
  asm volatile("cp.async.ca.shared.global [%0], [%1], 8;" ::"r"(d), "l"(gsrc) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
__device__ __forceinline__ void cp_async_wait_all() { asm volatile("cp.async.wait_all;" ::: "memory"); }

// ---- TMA bulk copies completing on an mbarrier ------------------------------
__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void fence_mbar_init() { asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory"); }
// one arrival that also expects `bytes` of transactions on the current phase
__device__ __forceinline__ void mbar_arrive_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes) : "memory");
}
// bulk global -> shared copy (16-B aligned, bytes a multiple of 16) signalling `bar`
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
               ::"r"(smem_u32(dst)), "l"(src), "r"(bytes), "r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  const uint32_t a = smem_u32(bar);
  uint32_t done = 0;
  while (!done) {
    asm volatile("{\n .reg .pred p;\n mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n selp.u32 %0, 1, 0, p;\n}"
                 : "=r"(done) : "r"(a), "r"(parity) : "memory");
  }
}

// ---- selector-form transition functions (see arb_internal.h) -------------
// x holds 4 states, one per byte (low nibble); returns the 4 images (bit 4 clear).
__device__ __forceinline__ uint32_t sel_apply4(Sel s, uint32_t x) {
  uint32_t out = 0;
#pragma unroll
  for (int j = 0; j < 4; ++j) {
    uint32_t src = (s >> (3 * j)) & 7u;
    uint32_t v = src < 4 ? (x >> src) & 0x01010101u : (src == 5 ? 0x01010101u : 0u);
    out |= v << j;
  }
  return out;
}
// ARB_F_BO contexts: bits 0-3 as sel_apply4, bit 4 (kCVp) kept, cleared or set
// by the selector's bits 12-13.
__device__ __forceinline__ uint32_t sel_apply5(Sel s, uint32_t x) {
  const uint32_t pop = (s >> 12) & 3u;
  return sel_apply4(s, x) | (pop == 0 ? (x & 0x10101010u) : (pop == 3 ? 0x10101010u : 0u));
}
// several accelerators (Z24): 8-output selectors on 8-bit states
__device__ __forceinline__ uint32_t sel8_apply4(uint32_t s, uint32_t x) {
  uint32_t out = 0;
#pragma unroll
  for (int j = 0; j < 8; ++j) {
    const uint32_t src = (s >> (4 * j)) & 15u;
    const uint32_t v = src < 8 ? (x >> src) & 0x01010101u : (src == 9 ? 0x01010101u : 0u);
    out |= v << j;
  }
  return out;
}
__device__ __forceinline__ uint32_t sel8_compose(uint32_t g, uint32_t f) {  // g after f
  uint32_t r = 0;
#pragma unroll
  for (int j = 0; j < 8; ++j) {
    const uint32_t gj = (g >> (4 * j)) & 15u;
    r |= (gj < 8 ? (f >> (4 * gj)) & 15u : gj) << (4 * j);
  }
  return r;
}
__device__ __forceinline__ Sel sel_compose(Sel g, Sel f) {  // g after f
  Sel r = (g & (3u << 12)) ? (g & (3u << 12)) : (f & (3u << 12));
#pragma unroll
  for (int j = 0; j < 4; ++j) {
    uint32_t gj = (g >> (3 * j)) & 7u;
    uint32_t v = gj < 4 ? (f >> (3 * gj)) & 7u : gj;
    r |= v << (3 * j);
  }
  return r;
}

}  // namespace arb
