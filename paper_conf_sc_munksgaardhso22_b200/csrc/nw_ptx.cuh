// nw_ptx.cuh — thin inline-PTX wrappers for sm_100a used by the wavefront kernel (nw_wave.cuh).
//
// Ref rows move from global to shared memory with 4-byte cp.async (LDGSTS; the rows are unaligned
// at the Rodinia pitch n+1) and the staging warp's L2 prefetch; the global border blocks with
// 16-byte cp.async.cg.  Staging <-> compute progress words are 8-byte release / acquire accesses
// at CTA scope.  The epoch-tagged border entries are polled with relaxed 8-byte loads (single-copy
// atomic for an aligned 8-byte access, PTX memory model) at GPU scope within a device and at
// system scope across NVLink peers, and prefetched a block at a time by 16-byte cp.async.cg (a
// weak read: DESIGN.md §4.4 states the hardware assumption it relies on); their stores live next
// to the kernel (nw_wave.cuh NW_ENT1 / NW_ENT2).
#pragma once
#include <cstdint>

namespace nwb200 {

__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
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
__device__ __forceinline__ void prefetch_l2_p(bool p, const void* a) {
  asm volatile("{ .reg .pred q; setp.ne.b32 q, %0, 0; @q prefetch.global.L2 [%1]; }" ::"r"(static_cast<int>(p)), "l"(a));
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
__device__ __forceinline__ unsigned ld_acquire_gpu_u32(const unsigned* p) {
  unsigned v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ uint64_t globaltimer_ns() {
  uint64_t t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}

}  // namespace nwb200
