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
// Square root of two values on the FMA pipe (no MUFU), for a fraction of the SDH's pairs when
// the XU pipe is the bound: a magic-constant reciprocal square root with one
// modified Newton step (constants of Moroz et al., |rel err| <= 6.5e-4), y = s r, then two
// Newton corrections y += (s - y^2) r / 2. 10 FP32 lane-ops + 2 ALU ops per value; max relative
// error 2^-24 over [1, 4) and the integers < 2^24 (exhaustive on the GPU: tools/sqrt_bound.cu),
// i.e. tighter than sqrt.approx. s = 0 gives 0; denormal s gives a value < 1e-19.
__device__ __forceinline__ float2 sqrt_sw2(float2 s) {
  float2 r = make_float2(__uint_as_float(0x5F1FFFF9u - (__float_as_uint(s.x) >> 1)),
                         __uint_as_float(0x5F1FFFF9u - (__float_as_uint(s.y) >> 1)));
  const float2 t = __fmul2_rn(s, r);
  const float2 u = __ffma2_rn(make_float2(-t.x, -t.y), r, make_float2(2.38924456f, 2.38924456f));
  r = __fmul2_rn(__fmul2_rn(r, make_float2(0.703952253f, 0.703952253f)), u);
  float2 y = __fmul2_rn(s, r);
  const float2 hr = __fmul2_rn(r, make_float2(0.5f, 0.5f));
  float2 e = __ffma2_rn(make_float2(-y.x, -y.y), y, s);
  y = __ffma2_rn(e, hr, y);
  e = __ffma2_rn(make_float2(-y.x, -y.y), y, s);
  return __ffma2_rn(e, hr, y);
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
