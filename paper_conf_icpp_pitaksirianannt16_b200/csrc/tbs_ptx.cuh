// tbs_ptx.cuh — thin inline-PTX wrappers for sm_100a used by the 2-BS kernels:
// mbarrier + cp.async.bulk (TMA 1-D bulk copy) for partner-tile staging, shared and
// global reductions for the output stage, MUFU square root.
#pragma once
#include <cstdint>

namespace tbs {

__device__ __forceinline__ uint32_t smem_addr(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

// ---- mbarrier --------------------------------------------------------------------
__device__ __forceinline__ void mbar_init(uint32_t bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(bar), "r"(count) : "memory");
}
__device__ __forceinline__ void fence_mbar_init() {
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx(uint32_t bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint32_t bar, uint32_t parity) {
  asm volatile(
      "{\n"
      ".reg .pred P1;\n"
      "TBS_WAIT:\n"
      "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n"
      "@P1 bra TBS_DONE;\n"
      "bra TBS_WAIT;\n"
      "TBS_DONE:\n"
      "}\n" ::"r"(bar),
      "r"(parity)
      : "memory");
}

// ---- TMA 1-D bulk copy global -> shared, completion counted on an mbarrier ----------
// dst, src 16-byte aligned, bytes a multiple of 16 (SASS: UBLKCP).
__device__ __forceinline__ void bulk_g2s(uint32_t dst, const void* src, uint32_t bytes, uint32_t bar) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(dst),
               "l"(src), "r"(bytes), "r"(bar)
               : "memory");
}

// ---- output-stage reductions -----------------------------------------------------
// Increment a u32 counter in shared memory (SASS: ATOMS.POPC.INC / ATOMS.ADD).
__device__ __forceinline__ void red_smem_inc(uint32_t addr) {
  asm volatile("red.shared.add.u32 [%0], 1;" ::"r"(addr));
}
// Same, predicated on (p > a) — the i<j / tail / row-range mask (one ISETP).
__device__ __forceinline__ void red_smem_inc_gt(uint32_t addr, int p, int a) {
  asm volatile(
      "{\n.reg .pred q;\n"
      "setp.gt.s32 q, %1, %2;\n"
      "@q red.shared.add.u32 [%0], 1;\n}\n" ::"r"(addr),
      "r"(p), "r"(a));
}
// Same, predicated on a computed condition (bucket-range passes).
__device__ __forceinline__ void red_smem_inc_if(uint32_t addr, bool c) {
  asm volatile(
      "{\n.reg .pred q;\n"
      "setp.ne.s32 q, %1, 0;\n"
      "@q red.shared.add.u32 [%0], 1;\n}\n" ::"r"(addr),
      "r"((int)c));
}
// Global u64 increment (partially privatised global histogram, SASS: REDG.E.ADD.64).
// System-scope u64 add (peer memory mapped over NVLink / CUDA IPC: the fused combine).
__device__ __forceinline__ void red_sys_add_u64(unsigned long long* addr, unsigned long long v) {
  asm volatile("red.relaxed.sys.global.add.u64 [%0], %1;" ::"l"(addr), "l"(v) : "memory");
}
__device__ __forceinline__ void red_gmem_inc64(unsigned long long* addr) {
  asm volatile("red.global.add.u64 [%0], 1;" ::"l"(addr) : "memory");
}
__device__ __forceinline__ void red_gmem_inc64_gt(unsigned long long* addr, int p, int a) {
  asm volatile(
      "{\n.reg .pred q;\n"
      "setp.gt.s32 q, %1, %2;\n"
      "@q red.global.add.u64 [%0], 1;\n}\n" ::"l"(addr),
      "r"(p), "r"(a)
      : "memory");
}

// ---- MUFU square root (max rel. error ~2^-23; DESIGN.md §Error budget) --------------
__device__ __forceinline__ float sqrt_approx(float x) {
  float r;
  asm("sqrt.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(x));
  return r;
}
__device__ __forceinline__ float ex2_approx(float x) {
  float r;
  asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(x));
  return r;
}

// Streaming (evict-first) 16-byte global store for the Type-III output.
__device__ __forceinline__ void st_cs_v4(float* p, float a, float b, float c, float d) {
  asm volatile("st.global.cs.v4.f32 [%0], {%1, %2, %3, %4};" ::"l"(p), "f"(a), "f"(b), "f"(c), "f"(d) : "memory");
}

}  // namespace tbs
