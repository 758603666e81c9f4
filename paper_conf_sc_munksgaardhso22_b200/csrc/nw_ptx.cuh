// nw_ptx.cuh — thin inline-PTX wrappers for sm_100a used by the NW kernels.
//
// Row segments move between global and shared memory with 16-byte cp.async (LDGSTS, completion
// on an mbarrier) and LDS.128/STG.128 (the per-row cp.async.bulk variants are kept for
// reference; small bulk copies serialise in the TMA unit).  Relaxed 64-bit loads/stores carry the epoch-tagged border entries (single-copy
// atomic for aligned 8-byte accesses, PTX memory model), at GPU scope within a device and at
// system scope across NVLink peers.
#pragma once
#include <cstdint>

namespace nwb200 {

__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

__device__ __forceinline__ int lds_s32(uint32_t a) {
  int v;
  asm volatile("ld.shared.b32 %0, [%1];" : "=r"(v) : "r"(a) : "memory");
  return v;
}
__device__ __forceinline__ void sts_s32(uint32_t a, int v) {
  asm volatile("st.shared.b32 [%0], %1;" ::"r"(a), "r"(v) : "memory");
}

// 16-byte asynchronous global->shared copy through L2 only (LDGSTS), and a 4-byte one
__device__ __forceinline__ void cp_async16(uint32_t dst, const void* src) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(dst), "l"(src) : "memory");
}
__device__ __forceinline__ void cp_async16_cg_p(bool p, uint32_t dst, const void* src) {
  asm volatile("{ .reg .pred q; setp.ne.b32 q, %0, 0; @q cp.async.cg.shared.global [%1], [%2], 16; }" ::"r"(static_cast<int>(p)),
               "r"(dst), "l"(src)
               : "memory");
}
__device__ __forceinline__ void cp_async4_p(bool p, uint32_t dst, const void* src) {
  asm volatile("{ .reg .pred q; setp.ne.b32 q, %0, 0; @q cp.async.ca.shared.global [%1], [%2], 4; }" ::"r"(static_cast<int>(p)),
               "r"(dst), "l"(src)
               : "memory");
}
__device__ __forceinline__ void cp_async4(uint32_t dst, const void* src) {
  asm volatile("cp.async.ca.shared.global [%0], [%1], 4;" ::"r"(dst), "l"(src) : "memory");
}
// arrive on `bar` once this thread's prior cp.async copies have landed (counts toward the
// arrival count given at init)
__device__ __forceinline__ void cp_async_arrive(uint32_t bar) {
  asm volatile("cp.async.mbarrier.arrive.noinc.shared::cta.b64 [%0];" ::"r"(bar) : "memory");
}
// predicated forms (no branch): p == false -> no access
__device__ __forceinline__ void cp_async16_p(bool p, uint32_t dst, const void* src) {
  asm volatile("{ .reg .pred q; setp.ne.b32 q, %0, 0; @q cp.async.cg.shared.global [%1], [%2], 16; }" ::"r"(static_cast<int>(p)),
               "r"(dst), "l"(src)
               : "memory");
}
__device__ __forceinline__ void prefetch_l2_p(bool p, const void* a) {
  asm volatile("{ .reg .pred q; setp.ne.b32 q, %0, 0; @q prefetch.global.L2 [%1]; }" ::"r"(static_cast<int>(p)), "l"(a));
}
__device__ __forceinline__ int4 lds128_p(bool p, uint32_t a) {
  int4 v = make_int4(0, 0, 0, 0);
  asm volatile("{ .reg .pred q; setp.ne.b32 q, %4, 0; @q ld.shared.v4.b32 {%0, %1, %2, %3}, [%5]; }"
               : "+r"(v.x), "+r"(v.y), "+r"(v.z), "+r"(v.w)
               : "r"(static_cast<int>(p)), "r"(a)
               : "memory");
  return v;
}
__device__ __forceinline__ void stg128_p(bool p, void* ptr, int4 v) {
  asm volatile("{ .reg .pred q; setp.ne.b32 q, %0, 0; @q st.global.v4.b32 [%1], {%2, %3, %4, %5}; }" ::"r"(static_cast<int>(p)),
               "l"(ptr), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w)
               : "memory");
}
__device__ __forceinline__ int lds32_p(bool p, uint32_t a) {
  int v = 0;
  asm volatile("{ .reg .pred q; setp.ne.b32 q, %1, 0; @q ld.shared.b32 %0, [%2]; }" : "+r"(v) : "r"(static_cast<int>(p)), "r"(a) : "memory");
  return v;
}
__device__ __forceinline__ void stg32_p(bool p, void* ptr, int v) {
  asm volatile("{ .reg .pred q; setp.ne.b32 q, %0, 0; @q st.global.b32 [%1], %2; }" ::"r"(static_cast<int>(p)), "l"(ptr), "r"(v)
               : "memory");
}
__device__ __forceinline__ int4 lds128(uint32_t a) {
  int4 v;
  asm volatile("ld.shared.v4.b32 {%0, %1, %2, %3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "r"(a) : "memory");
  return v;
}
__device__ __forceinline__ void stg128(void* p, int4 v) {
  asm volatile("st.global.v4.b32 [%0], {%1, %2, %3, %4};" ::"l"(p), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w) : "memory");
}

__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_async_wait() {
  asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory");
}
// staging -> compute progress word {lo, hi} with release / acquire semantics at CTA scope
__device__ __forceinline__ void st_release_cta_v2(uint32_t a, uint32_t lo, uint32_t hi) {
  asm volatile("{ .reg .b64 e; mov.b64 e, {%1, %2}; st.release.cta.shared.b64 [%0], e; }" ::"r"(a), "r"(lo), "r"(hi) : "memory");
}
__device__ __forceinline__ uint64_t ld_acquire_cta(uint32_t a) {
  uint64_t v;
  asm volatile("ld.acquire.cta.shared.b64 %0, [%1];" : "=l"(v) : "r"(a) : "memory");
  return v;
}

__device__ __forceinline__ void mbar_init(uint32_t bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(bar), "r"(count) : "memory");
}
__device__ __forceinline__ void fence_mbar_init() {
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void mbar_arrive(uint32_t bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(bar) : "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx(uint32_t bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes)
               : "memory");
}
__device__ __forceinline__ bool mbar_try_wait(uint32_t bar, uint32_t parity) {
  uint32_t ok;
  asm volatile(
      "{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0, 1, 0, p; }"
      : "=r"(ok)
      : "r"(bar), "r"(parity)
      : "memory");
  return ok != 0;
}
__device__ __forceinline__ void mbar_wait(uint32_t bar, uint32_t parity) {
  while (!mbar_try_wait(bar, parity)) {
  }
}

// global -> shared bulk copy, completion reported to `bar` as transaction bytes.
__device__ __forceinline__ void bulk_g2s(uint32_t dst, const void* src, uint32_t bytes, uint32_t bar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(dst),
      "l"(src), "r"(bytes), "r"(bar)
      : "memory");
}
// shared -> global bulk copy in the executing thread's current bulk group.
__device__ __forceinline__ void bulk_s2g(void* dst, uint32_t src, uint32_t bytes) {
  asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(dst), "r"(src), "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void bulk_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void bulk_wait_read() {
  asm volatile("cp.async.bulk.wait_group.read %0;" ::"n"(N) : "memory");
}
template <int N>
__device__ __forceinline__ void bulk_wait_all() {
  asm volatile("cp.async.bulk.wait_group %0;" ::"n"(N) : "memory");
}
// generic-proxy shared-memory accesses -> visible to / ordered with the async proxy.
__device__ __forceinline__ void fence_proxy_async() {
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}

__device__ __forceinline__ uint64_t ld_relaxed_gpu(const uint64_t* p) {
  uint64_t v;
  asm volatile("ld.relaxed.gpu.global.b64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ uint64_t ld_relaxed_sys(const uint64_t* p) {
  uint64_t v;
  asm volatile("ld.relaxed.sys.global.b64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_relaxed_gpu(uint64_t* p, uint64_t v) {
  asm volatile("st.relaxed.gpu.global.b64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ void st_relaxed_sys(uint64_t* p, uint64_t v) {
  asm volatile("st.relaxed.sys.global.b64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
// (lo, hi) as one 64-bit single-copy-atomic store: the epoch-tagged border entry {value, epoch}
__device__ __forceinline__ void st_relaxed_gpu_v2(uint64_t* p, uint32_t lo, uint32_t hi) {
  asm volatile("{ .reg .b64 e; mov.b64 e, {%1, %2}; st.relaxed.gpu.global.b64 [%0], e; }" ::"l"(p), "r"(lo), "r"(hi)
               : "memory");
}
__device__ __forceinline__ void st_relaxed_sys_v2(uint64_t* p, uint32_t lo, uint32_t hi) {
  asm volatile("{ .reg .b64 e; mov.b64 e, {%1, %2}; st.relaxed.sys.global.b64 [%0], e; }" ::"l"(p), "r"(lo), "r"(hi)
               : "memory");
}
__device__ __forceinline__ uint64_t globaltimer_ns() {
  uint64_t t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}

}  // namespace nwb200
