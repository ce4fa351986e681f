// ptx.cuh — sm_100a load/store primitives with explicit cache policies.
#pragma once
#include <stdint.h>

namespace inl {

// 256-bit streaming load (LDG.E.NA.EFL2.256): CSR col_idx / val are read once per
// call, so they bypass L1 and are marked evict-first in L2, which keeps the
// gathered vector (x, PageRank contributions) resident in the 126 MB L2.
struct U32x8 {
  uint32_t v[8];
};

__device__ __forceinline__ U32x8 ld_stream_256(const void *p) {
  U32x8 r;
  asm volatile(
      "ld.global.nc.L1::no_allocate.L2::evict_first.v8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
      : "=r"(r.v[0]), "=r"(r.v[1]), "=r"(r.v[2]), "=r"(r.v[3]), "=r"(r.v[4]), "=r"(r.v[5]),
        "=r"(r.v[6]), "=r"(r.v[7])
      : "l"(p));
  return r;
}

__device__ __forceinline__ uint32_t ld_stream_32(const void *p) {
  uint32_t r;
  asm volatile("ld.global.nc.L1::no_allocate.b32 %0, [%1];" : "=r"(r) : "l"(p));
  return r;
}


// Streaming 32-bit load with an L2 eviction policy (createpolicy), no L1 allocation.
__device__ __forceinline__ uint32_t ld_stream_pol(const void *p, uint64_t pol) {
  uint32_t r;
  asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.b32 %0, [%1], %2;" : "=r"(r) : "l"(p), "l"(pol));
  return r;
}

// fire-and-forget global reductions (RED: the issuing warp never waits for a result)
__device__ __forceinline__ void red_min_u32(uint32_t *p, uint32_t v) {
  asm volatile("red.relaxed.gpu.global.min.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ void red_or_b32(uint32_t *p, uint32_t v) {
  asm volatile("red.relaxed.gpu.global.or.b32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

__device__ __forceinline__ uint64_t policy_evict_last() {
  uint64_t p;
  asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
  return p;
}

// Predicated gather (no branch): r = pred ? *p : 0.  Read-only path, L2 evict-last.
__device__ __forceinline__ float ld_gather_pred(const float *p, bool pred, uint64_t pol) {
  float r = 0.0f;
  asm("{ .reg .pred q; setp.ne.b32 q, %2, 0; @q ld.global.nc.L2::cache_hint.f32 %0, [%1], %3; }"
      : "+f"(r)
      : "l"(p), "r"((int)pred), "l"(pol));
  return r;
}

__device__ __forceinline__ uint32_t ld_stream_pred(const void *p, bool pred) {
  uint32_t r = 0;
  asm("{ .reg .pred q; setp.ne.b32 q, %2, 0; @q ld.global.nc.L1::no_allocate.b32 %0, [%1]; }"
      : "+r"(r)
      : "l"(p), "r"((int)pred));
  return r;
}

// Gather of the dense vector: read-only path, L2 evict-last.
__device__ __forceinline__ float ld_gather_f32(const float *p, uint64_t pol) {
  float r;
  asm volatile("ld.global.nc.L2::cache_hint.f32 %0, [%1], %2;" : "=f"(r) : "l"(p), "l"(pol));
  return r;
}

__device__ __forceinline__ float warp_sum(float v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  return v;
}

__device__ __forceinline__ double warp_sum_d(double v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  return v;
}

}  // namespace inl

// ---- TMA bulk copies + mbarriers (sm_90+/sm_100a async proxy) ----------------------------
namespace inl {

__device__ __forceinline__ uint32_t smem_u32(const void *p) {
  return (uint32_t)__cvta_generic_to_shared(p);
}

__device__ __forceinline__ void mbar_init(uint64_t *bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}

__device__ __forceinline__ void fence_mbar_init() {
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}

__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t *bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes)
               : "memory");
}

__device__ __forceinline__ void mbar_arrive(uint64_t *bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}

__device__ __forceinline__ void mbar_wait(uint64_t *bar, uint32_t parity) {
  uint32_t done = 0;
  do {
    asm volatile(
        "{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0, 1, 0, p; }"
        : "=r"(done)
        : "r"(smem_u32(bar)), "r"(parity)
        : "memory");
  } while (!done);
}

__device__ __forceinline__ uint64_t policy_evict_first() {
  uint64_t p;
  asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
  return p;
}

// 1-D bulk copy global -> shared (UBLKCP), completion counted on `bar` in bytes.
// dst/src 16-byte aligned, bytes a multiple of 16.
__device__ __forceinline__ void bulk_g2s(void *dst, const void *src, uint32_t bytes, uint64_t *bar,
                                         uint64_t pol) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;"
      ::"r"(smem_u32(dst)), "l"(src), "r"(bytes), "r"(smem_u32(bar)), "l"(pol)
      : "memory");
}

__device__ __forceinline__ void fence_proxy_async_smem() {
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}

// Named barrier among the `n` consumer threads (id 1; id 0 is __syncthreads).
__device__ __forceinline__ void consumer_sync(int n) {
  asm volatile("bar.sync 1, %0;" ::"r"(n) : "memory");
}

}  // namespace inl

namespace inl {
// TMA bulk prefetch of [p, p + bytes) into L2 (fire and forget; p, bytes 16-B aligned).
__device__ __forceinline__ void bulk_prefetch_l2(const void *p, uint32_t bytes) {
  asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(p), "r"(bytes) : "memory");
}

// Prefetch elements [lo, hi) of an array ending at `end` (clamped, 16-B aligned).
__device__ __forceinline__ void prefetch_span(const void *lo, const void *hi, const void *end) {
  uintptr_t a = (uintptr_t)lo & ~(uintptr_t)15, b = ((uintptr_t)hi + 15) & ~(uintptr_t)15;
  const uintptr_t c = (uintptr_t)end & ~(uintptr_t)15;
  if (b > c) b = c;
  if (b > a) bulk_prefetch_l2((const void *)a, (uint32_t)(b - a));
}
}  // namespace inl
