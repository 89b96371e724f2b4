// lpt_util.cuh — small PTX helpers shared by the lane-per-trace replay
// kernels (replay_lpt.cu, replay_lpt16.cu): predicated cp.async / st.shared,
// clamped shifts and 64-bit mask bit operations.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

namespace convgpu {
namespace lpt {

__device__ __forceinline__ uint32_t smem_addr(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void cp_async4(uint32_t* dst, const uint32_t* src) {
  asm volatile("cp.async.ca.shared.global [%0], [%1], 4;" ::"r"(smem_addr(dst)), "l"(src) : "memory");
}
// predicated forms (one predicated instruction, no divergent branch)
__device__ __forceinline__ void cp_async4_if(uint32_t* dst, const uint32_t* src, bool on) {
  asm volatile("{ .reg .pred q; setp.ne.u32 q, %2, 0; @q cp.async.ca.shared.global [%0], [%1], 4; }"
               ::"r"(smem_addr(dst)), "l"(src), "r"((uint32_t)on) : "memory");
}
__device__ __forceinline__ void cp_wait0_if(bool on) {
  asm volatile("{ .reg .pred q; setp.ne.u32 q, %0, 0; @q cp.async.wait_group 0; }" ::"r"((uint32_t)on) : "memory");
}
__device__ __forceinline__ void sts_if(uint32_t* dst, uint32_t v, bool on) {  // predicated st.shared
  asm volatile("{ .reg .pred q; setp.ne.u32 q, %2, 0; @q st.shared.u32 [%0], %1; }"
               ::"r"(smem_addr(dst)), "r"(v), "r"((uint32_t)on) : "memory");
}
__device__ __forceinline__ void cp_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
__device__ __forceinline__ void cp_wait1() { asm volatile("cp.async.wait_group 1;" ::: "memory"); }
__device__ __forceinline__ void cp_wait0() { asm volatile("cp.async.wait_group 0;" ::: "memory"); }

// PTX shifts clamp: a shift by >= 32 gives 0 (no guard instructions, unlike
// C++ where it is undefined); b - 32 wraps to a huge count for b < 32.
__device__ __forceinline__ uint32_t shl_c(uint32_t v, uint32_t s) {
  uint32_t r;
  asm("shl.b32 %0, %1, %2;" : "=r"(r) : "r"(v), "r"(s));
  return r;
}
__device__ __forceinline__ uint32_t shr_c(uint32_t v, uint32_t s) {
  uint32_t r;
  asm("shr.b32 %0, %1, %2;" : "=r"(r) : "r"(v), "r"(s));
  return r;
}
__device__ __forceinline__ bool bit64(uint32_t lo, uint32_t hi, uint32_t b) {  // b < 64
  return ((shr_c(lo, b) | shr_c(hi, b - 32u)) & 1u) != 0;
}
__device__ __forceinline__ void set64(uint32_t& lo, uint32_t& hi, uint32_t b, bool on) {  // b < 64
  const uint32_t ml = shl_c(1u, b), mh = shl_c(1u, b - 32u);
  lo = on ? (lo | ml) : (lo & ~ml);
  hi = on ? (hi | mh) : (hi & ~mh);
}
__device__ __forceinline__ uint32_t ffs64(uint32_t lo, uint32_t hi) {  // lowest set bit, 64 if none
  const uint32_t a = (uint32_t)__ffs(lo), b = (uint32_t)__ffs(hi);  // both always: no branch
  return a ? a - 1u : (b ? b + 31u : 64u);
}
__device__ __forceinline__ uint32_t fls64(uint32_t lo, uint32_t hi) {  // highest set bit
  return hi ? 63u - (uint32_t)__clz(hi) : 31u - (uint32_t)__clz(lo);
}
// position of the j-th (0-based) set bit of (hi:lo), j < popc: a branch-free
// popc binary search (the __fns intrinsic is a branchy software sequence,
// and two of them behind a lo/hi branch diverge inside a warp)
__device__ __forceinline__ uint32_t nth_set64(uint32_t lo, uint32_t hi, uint32_t j) {
  const uint32_t cl = (uint32_t)__popc(lo);
  const bool up = j >= cl;
  uint32_t w = up ? hi : lo, pos = up ? 32u : 0u;
  j -= up ? cl : 0u;
#pragma unroll
  for (uint32_t s = 16; s >= 1; s >>= 1) {
    const uint32_t c = (uint32_t)__popc(w & ((1u << s) - 1u));
    const bool b = j >= c;
    j -= b ? c : 0u;
    pos += b ? s : 0u;
    w = b ? (w >> s) : w;
  }
  return pos;
}
__device__ __forceinline__ void lowmask64(uint32_t r, uint32_t& lo, uint32_t& hi) {  // bits < r
  lo = r >= 32 ? 0xFFFFFFFFu : ((1u << r) - 1u);
  hi = r >= 64 ? 0xFFFFFFFFu : (r <= 32 ? 0u : ((1u << (r - 32)) - 1u));
}

// ---- tensor memory (TMEM) as per-thread spill space ------------------------
// The lane-per-trace kernels keep statically indexed per-trace arrays (e.g.
// arrival + sum of deltas of every container) from a trace's init to its
// epilogue.  In registers they would pin 64 registers across the whole event
// loop; instead each thread parks them in its own TMEM lane (warp w of the
// CTA owns lanes 32 * (w % 4) .. + 31, shape 32x32b: one 32-bit column
// element per thread) with tcgen05.st and reads them back with tcgen05.ld.
// All of these are .sync.aligned: every lane of the warp executes them,
// converged, with the same address.
__device__ __forceinline__ void tmem_alloc(uint32_t* smem_dst, uint32_t ncols) {  // one warp
  asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;"
               ::"r"(smem_addr(smem_dst)), "r"(ncols) : "memory");
  asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
}
__device__ __forceinline__ void tmem_dealloc(uint32_t taddr, uint32_t ncols) {  // the same warp
  asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(taddr), "r"(ncols) : "memory");
}
__device__ __forceinline__ void tmem_fence_before_sync() {
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
}
__device__ __forceinline__ void tmem_fence_after_sync() {
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
}
// 16 consecutive columns of this thread's lane.  No "memory" clobber: TMEM is
// not generic memory, so global / shared accesses may be scheduled across the
// store (init's loads of the next containers overlap it); tcgen05.wait::st and
// the volatile loads keep TMEM ordered.
#ifndef TMEM_ST_CLOBBER
#define TMEM_ST_CLOBBER
#endif
__device__ __forceinline__ void tmem_st16(uint32_t taddr, const uint32_t* v) {
  asm volatile(
      "tcgen05.st.sync.aligned.32x32b.x16.b32 [%0], {%1, %2, %3, %4, %5, %6, %7, %8, %9, %10, %11, "
      "%12, %13, %14, %15, %16};"
      ::"r"(taddr), "r"(v[0]), "r"(v[1]), "r"(v[2]), "r"(v[3]), "r"(v[4]), "r"(v[5]), "r"(v[6]),
        "r"(v[7]), "r"(v[8]), "r"(v[9]), "r"(v[10]), "r"(v[11]), "r"(v[12]), "r"(v[13]),
        "r"(v[14]), "r"(v[15])
      TMEM_ST_CLOBBER);
}
__device__ __forceinline__ void tmem_ld16(uint32_t taddr, uint32_t* v) {
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0, %1, %2, %3, %4, %5, %6, %7, %8, %9, %10, %11, "
      "%12, %13, %14, %15}, [%16];"
      : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]),
        "=r"(v[7]), "=r"(v[8]), "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]),
        "=r"(v[14]), "=r"(v[15])
      : "r"(taddr)
      : "memory");
}
// 16-byte global loads issued exactly where written (volatile: the compiler
// may not sink them to their first use, so a batch of them is in flight
// together), cached at L2 only (.cg): one warp's 32 traces are 32 different
// lines per load, so L1 (what shared memory leaves of it) cannot hold them,
// while L2 keeps the rows for the event loop's op fetches.  Measured on the
// compact kernel's init: .cg 4.31, .nc 4.24, .ca 4.22, .cs (evict-first) 3.28
// x 10^10 events/s.
__device__ __forceinline__ uint4 ldg4_cg(const void* p) {
  uint4 v;
  asm volatile("ld.global.cg.v4.u32 {%0, %1, %2, %3}, [%4];"
               : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p));
  return v;
}
// 32-byte load (LDG.256, sm_100): 8 words, the address 32-B aligned
__device__ __forceinline__ void ldg8_cg(uint32_t (&v)[8], const void* p) {
  asm volatile("ld.global.cg.v8.u32 {%0, %1, %2, %3, %4, %5, %6, %7}, [%8];"
               : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]),
                 "=r"(v[7])
               : "l"(p));
}
// 32-byte / 8-byte streaming (evict-first) stores, 32- / 8-B aligned
__device__ __forceinline__ void stg8_cs(void* p, const uint32_t (&v)[8]) {
  asm volatile("st.global.cs.v8.u32 [%0], {%1, %2, %3, %4, %5, %6, %7, %8};"
               ::"l"(p), "r"(v[0]), "r"(v[1]), "r"(v[2]), "r"(v[3]), "r"(v[4]), "r"(v[5]), "r"(v[6]),
                 "r"(v[7]) : "memory");
}
__device__ __forceinline__ void stg2_cs(void* p, uint32_t a, uint32_t b) {
  asm volatile("st.global.cs.v2.u32 [%0], {%1, %2};" ::"l"(p), "r"(a), "r"(b) : "memory");
}
__device__ __forceinline__ void tmem_wait_st() { asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory"); }
__device__ __forceinline__ void tmem_wait_ld() { asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory"); }

}  // namespace lpt
}  // namespace convgpu
