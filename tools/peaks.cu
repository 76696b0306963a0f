// Microbenchmarks for the pipe peaks that bound the 2-BS hot path on sm_100a
// (SURVEY.md §8(d) "Microbenchmarks that define the peaks").
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/peaks tools/peaks.cu
// Prints one JSON object: per-op lane-ops/s, lane-ops/clk/SM, and the SM clock seen.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e_ = (x); if (e_ != cudaSuccess) { \
  fprintf(stderr, "%s:%d %s\n", __FILE__, __LINE__, cudaGetErrorString(e_)); return 1; } } while (0)

constexpr int ITERS = 4096;

// ---- clock probe: SM cycles vs ns over a busy loop -------------------------
__global__ void k_clock(unsigned long long* out, int spin) {
  unsigned long long c0 = clock64(), t0, t1;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
  float x = threadIdx.x;
  for (int i = 0; i < spin; ++i) x = fmaf(x, 0.999f, 0.5f);
  unsigned long long c1 = clock64();
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t1));
  if (threadIdx.x == 0) { out[2 * blockIdx.x] = c1 - c0; out[2 * blockIdx.x + 1] = t1 - t0; }
  if (x == -1.f) out[0] = 0;
}

// ---- FP32 scalar FFMA, all-register operands ------------------------------
__global__ void k_ffma(float* out, float y0, float z0) {
  float y = y0 + threadIdx.x * 1e-9f, z = z0 - threadIdx.x * 1e-9f;
  float x[8];
#pragma unroll
  for (int c = 0; c < 8; ++c) x[c] = threadIdx.x + c;
  for (int i = 0; i < ITERS; ++i) {
#pragma unroll
    for (int c = 0; c < 8; ++c) x[c] = fmaf(x[c], y, z);
  }
  float s = 0; for (int c = 0; c < 8; ++c) s += x[c];
  if (s == 1.2345f) out[0] = s;
}

// ---- FP32 packed FFMA2 (fma.rn.f32x2) ---------------------------------------
__global__ void k_ffma2(float* out, float y0, float z0) {
  float2 y = make_float2(y0 + threadIdx.x * 1e-9f, y0), z = make_float2(z0, z0 - threadIdx.x * 1e-9f);
  float2 x[8];
#pragma unroll
  for (int c = 0; c < 8; ++c) x[c] = make_float2(threadIdx.x + c, c);
  for (int i = 0; i < ITERS; ++i) {
#pragma unroll
    for (int c = 0; c < 8; ++c) x[c] = __ffma2_rn(x[c], y, z);
  }
  float s = 0; for (int c = 0; c < 8; ++c) s += x[c].x + x[c].y;
  if (s == 1.2345f) out[0] = s;
}

// ---- packed FFMA2 and scalar FFMA interleaved on independent chains: does the scalar
// stream use capacity (fmalite) the packed one leaves idle? Lane-ops = 2 x FFMA2 + FFMA.
__global__ void k_mix(float* out, float y0, float z0) {
  float2 y = make_float2(y0 + threadIdx.x * 1e-9f, y0), z = make_float2(z0, z0 - threadIdx.x * 1e-9f);
  float2 x[4];
  float w[4];
#pragma unroll
  for (int c = 0; c < 4; ++c) { x[c] = make_float2(threadIdx.x + c, c); w[c] = threadIdx.x - c; }
  for (int i = 0; i < ITERS; ++i) {
#pragma unroll
    for (int c = 0; c < 4; ++c) {
      x[c] = __ffma2_rn(x[c], y, z);
      w[c] = fmaf(w[c], y.x, z.y);
    }
  }
  float s = 0; for (int c = 0; c < 4; ++c) s += x[c].x + x[c].y + w[c];
  if (s == 1.2345f) out[0] = s;
}

// ---- the SDH distance stream: FADD2 with a broadcast scalar operand (a - p for two anchors)
// then FFMA2 squares, as in run_chunk. Lane-ops = 2 per packed instruction.
__global__ void k_dist(float* out, float p0) {
  float2 a[4], s[4];
#pragma unroll
  for (int c = 0; c < 4; ++c) { a[c] = make_float2(threadIdx.x * 1e-3f + c, c * 0.5f); s[c] = make_float2(0.f, 0.f); }
  float p = p0 + threadIdx.x * 1e-7f;
  for (int i = 0; i < ITERS; ++i) {
#pragma unroll
    for (int c = 0; c < 4; ++c) {
      const float2 d = __fadd2_rn(a[c], make_float2(p, p));
      s[c] = __ffma2_rn(d, d, s[c]);
    }
    p += 1e-6f;
  }
  float t = 0; for (int c = 0; c < 4; ++c) t += s[c].x + s[c].y;
  if (t == 1.2345f) out[0] = t;
}

// ---- FP32 scalar FADD / packed FADD2 ----------------------------------------
__global__ void k_fadd(float* out, float y0) {
  float y = y0 + threadIdx.x * 1e-9f;
  float x[8];
#pragma unroll
  for (int c = 0; c < 8; ++c) x[c] = threadIdx.x + c;
  for (int i = 0; i < ITERS; ++i) {
#pragma unroll
    for (int c = 0; c < 8; ++c) x[c] = x[c] - y;
  }
  float s = 0; for (int c = 0; c < 8; ++c) s += x[c];
  if (s == 1.2345f) out[0] = s;
}
__global__ void k_fadd2(float* out, float y0) {
  float2 y = make_float2(y0 + threadIdx.x * 1e-9f, y0);
  float2 x[8];
#pragma unroll
  for (int c = 0; c < 8; ++c) x[c] = make_float2(threadIdx.x + c, c);
  for (int i = 0; i < ITERS; ++i) {
#pragma unroll
    for (int c = 0; c < 8; ++c) x[c] = __fadd2_rn(x[c], y);
  }
  float s = 0; for (int c = 0; c < 8; ++c) s += x[c].x + x[c].y;
  if (s == 1.2345f) out[0] = s;
}

// ---- MUFU: sqrt.approx / rsqrt.approx / ex2.approx ---------------------------
template <int OP>
__global__ void k_mufu(float* out) {
  float x[8];
#pragma unroll
  for (int c = 0; c < 8; ++c) x[c] = 1.5f + threadIdx.x * 1e-3f + c;
  for (int i = 0; i < ITERS; ++i) {
#pragma unroll
    for (int c = 0; c < 8; ++c) {
      if (OP == 0) asm volatile("sqrt.approx.f32 %0, %0;" : "+f"(x[c]));
      if (OP == 1) asm volatile("rsqrt.approx.f32 %0, %0;" : "+f"(x[c]));
      if (OP == 2) asm volatile("ex2.approx.f32 %0, %0;" : "+f"(x[c]));
    }
  }
  float s = 0; for (int c = 0; c < 8; ++c) s += x[c];
  if (s == 1.2345f) out[0] = s;
}

// ---- shared-memory atomics ---------------------------------------------------
// MODE 0: lane-private rows (word 32*k + lane): no bank conflict, no same address.
// MODE 1: one copy of 256 bins, pseudo-random bin per lane (random bank conflicts).
// MODE 2: all lanes of a warp hit one address.
template <int MODE>
__global__ void k_atoms(unsigned* out) {
  extern __shared__ unsigned h[];
  const int lane = threadIdx.x & 31;
  for (int i = threadIdx.x; i < 64 * 32; i += blockDim.x) h[i] = 0;
  __syncthreads();
  unsigned k[8];
#pragma unroll
  for (int c = 0; c < 8; ++c) k[c] = (threadIdx.x * 2654435761u) ^ (c * 40503u);
  unsigned* base = h + lane;
  for (int i = 0; i < ITERS / 4; ++i) {
#pragma unroll
    for (int c = 0; c < 8; ++c) {
      k[c] = k[c] * 1664525u + 1013904223u;
      if (MODE == 0) atomicAdd(base + ((k[c] >> 26) << 5), 1u);
      if (MODE == 1) atomicAdd(h + (k[c] >> 24), 1u);
      if (MODE == 2) atomicAdd(h + (c << 5), 1u);
    }
  }
  __syncthreads();
  if (threadIdx.x == 0 && h[5] == 0xffffffffu) out[0] = h[0];
}

// Pure shared atomics: 8 fixed lane-private addresses per thread, no ALU per atomic.
__global__ void k_atoms_pure(unsigned* out) {
  extern __shared__ unsigned h[];
  const int lane = threadIdx.x & 31;
  for (int i = threadIdx.x; i < 64 * 32; i += blockDim.x) h[i] = 0;
  __syncthreads();
  uint32_t a[8];
#pragma unroll
  for (int c = 0; c < 8; ++c)
    a[c] = (uint32_t)__cvta_generic_to_shared(h + ((threadIdx.x * 7 + c * 13) & 63) * 32 + lane);
  for (int i = 0; i < ITERS / 4; ++i) {
#pragma unroll
    for (int c = 0; c < 8; ++c) asm volatile("red.shared.add.u32 [%0], 1;" ::"r"(a[c]));
  }
  __syncthreads();
  if (threadIdx.x == 0 && h[5] == 0xffffffffu) out[0] = h[0];
}

// Random bins over a LARGE histogram (16384 bins), R replicas per bin laid out
// word[k * R + (lane & (R-1))] exactly as SdhSmemOp<LOG2R>: the bank of a lane's increment is
// random, so a warp's ATOMS costs max-bank-load wavefronts. Occupancy set by the launch.
template <int LOG2R>
__global__ void k_atoms_big(unsigned* out, int log2bins) {
  extern __shared__ unsigned h[];
  const int lane = threadIdx.x & 31;
  const int words = (1 << log2bins) << LOG2R;
  for (int i = threadIdx.x; i < words; i += blockDim.x) h[i] = 0;
  __syncthreads();
  unsigned k[8];
#pragma unroll
  for (int c = 0; c < 8; ++c) k[c] = (threadIdx.x * 2654435761u + blockIdx.x * 97u) ^ (c * 40503u);
  const uint32_t base = (uint32_t)__cvta_generic_to_shared(h) + (uint32_t)((lane & ((1 << LOG2R) - 1)) * 4);
  const int sh = 32 - log2bins;
  for (int i = 0; i < ITERS / 4; ++i) {
#pragma unroll
    for (int c = 0; c < 8; ++c) {
      k[c] = k[c] * 1664525u + 1013904223u;
      asm volatile("red.shared.add.u32 [%0], 1;" ::"r"(base + ((k[c] >> sh) << (LOG2R + 2))));
    }
  }
  __syncthreads();
  if (threadIdx.x == 0 && h[5] == 0xffffffffu) out[0] = h[0];
}

// Same-address degree: groups of DEG lanes share one word of a warp-uniform row (32/DEG
// distinct addresses per warp instruction, all in distinct banks). (Bank-conflict degree DEG,
// DEG distinct rows hit through one bank: k_atoms_bank.)
template <int DEG>
__global__ void k_atoms_deg(unsigned* out) {
  extern __shared__ unsigned h[];
  const int lane = threadIdx.x & 31;
  for (int i = threadIdx.x; i < 64 * 32; i += blockDim.x) h[i] = 0;
  __syncthreads();
  uint32_t a[8];
#pragma unroll
  for (int c = 0; c < 8; ++c)
    a[c] = (uint32_t)__cvta_generic_to_shared(h + (((threadIdx.x >> 5) * 7 + c * 13) & 63) * 32 + (lane & ~(DEG - 1)));
  for (int i = 0; i < ITERS / 4; ++i) {
#pragma unroll
    for (int c = 0; c < 8; ++c) asm volatile("red.shared.add.u32 [%0], 1;" ::"r"(a[c]));
  }
  __syncthreads();
  if (threadIdx.x == 0 && h[5] == 0xffffffffu) out[0] = h[0];
}

template <int DEG>
__global__ void k_atoms_bank(unsigned* out) {
  extern __shared__ unsigned h[];
  const int lane = threadIdx.x & 31;
  for (int i = threadIdx.x; i < 64 * 32; i += blockDim.x) h[i] = 0;
  __syncthreads();
  uint32_t a[8];
#pragma unroll
  for (int c = 0; c < 8; ++c)   // lanes of a group: the same bank (column), different rows
    a[c] = (uint32_t)__cvta_generic_to_shared(h + (((threadIdx.x >> 5) * 7 + c * 13 + (lane & (DEG - 1))) & 63) * 32 +
                                              (lane & ~(DEG - 1)));
  for (int i = 0; i < ITERS / 4; ++i) {
#pragma unroll
    for (int c = 0; c < 8; ++c) asm volatile("red.shared.add.u32 [%0], 1;" ::"r"(a[c]));
  }
  __syncthreads();
  if (threadIdx.x == 0 && h[5] == 0xffffffffu) out[0] = h[0];
}

// ---- float -> int conversion (F2I: to confirm it must be avoided per pair) --
__global__ void k_f2i(float* out) {
  float x[8];
  int acc = 0;
#pragma unroll
  for (int c = 0; c < 8; ++c) x[c] = 1.5f + threadIdx.x * 1e-3f + c;
  for (int i = 0; i < ITERS; ++i) {
#pragma unroll
    for (int c = 0; c < 8; ++c) {
      int k;
      asm volatile("cvt.rmi.s32.f32 %0, %1;" : "=r"(k) : "f"(x[c]));
      acc ^= k;
      x[c] += 0.75f;   // a new operand every iteration (FADD on the FMA pipe, beside the conversion)
    }
  }
  if (acc == 12345) out[0] = (float)acc;
}

// ---- SHFL (the paper's Alg. 4 register sharing moves partners by shuffles) -------------------
__global__ void k_shfl(float* out) {
  float v[8];
#pragma unroll
  for (int c = 0; c < 8; ++c) v[c] = threadIdx.x + c;
  for (int i = 0; i < ITERS; ++i) {
#pragma unroll
    for (int c = 0; c < 8; ++c) v[c] = __shfl_xor_sync(0xffffffffu, v[c], 1 << (c & 3));   // data stays lane-varying
  }
  float s = 0; for (int c = 0; c < 8; ++c) s += v[c];
  if (s == 1.2345f) out[0] = s;
}

// ---- LDS.128 broadcast ---------------------------------------------------------
__global__ void k_lds128(float* out) {
  __shared__ float4 s[1024];
  for (int i = threadIdx.x; i < 1024; i += blockDim.x) s[i] = make_float4(i, i + 1, i + 2, i + 3);
  __syncthreads();
  float4 a = make_float4(0, 0, 0, 0);
  for (int i = 0; i < ITERS; ++i) {
    float4 v = s[(i * 8) & 1023];
    a.x += v.x; a.y += v.y; a.z += v.z; a.w += v.w;
  }
  if (a.x + a.y + a.z + a.w == 1.2345f) out[0] = a.x;
}

// ---- HBM streaming write (st.global.cs.v4) --------------------------------------
__global__ void k_write(float4* __restrict__ dst, size_t n4) {
  size_t stride = (size_t)gridDim.x * blockDim.x;
  float4 v = make_float4(threadIdx.x, 1.f, 2.f, 3.f);
  for (size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x; i < n4; i += stride) __stcs(dst + i, v);
}

int main() {
  cudaDeviceProp p; CK(cudaGetDeviceProperties(&p, 0));
  const int sms = p.multiProcessorCount;
  float* dout; CK(cudaMalloc(&dout, 1 << 20));
  unsigned long long* dclk; CK(cudaMalloc(&dclk, 2 * 8 * sms * sizeof(unsigned long long)));
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  const int threads = 256, blocks = sms * 8;   // 64 warps / SM
  auto timeit = [&](auto launch) -> double {
    launch(); cudaDeviceSynchronize();
    cudaEventRecord(e0); for (int r = 0; r < 5; ++r) launch(); cudaEventRecord(e1);
    cudaEventSynchronize(e1); float ms; cudaEventElapsedTime(&ms, e0, e1); return ms / 5 * 1e-3;
  };
  // clock
  k_clock<<<sms, 128>>>(dclk, 1 << 22); CK(cudaDeviceSynchronize());
  unsigned long long hclk[2]; CK(cudaMemcpy(hclk, dclk, sizeof(hclk), cudaMemcpyDeviceToHost));
  double mhz = (double)hclk[0] / (double)hclk[1] * 1e3;
  const double thr = (double)blocks * threads;
  printf("{\"gpu\": \"%s\", \"sms\": %d, \"clock_mhz_busy\": %.1f", p.name, sms, mhz);
  auto rep = [&](const char* name, double lane_ops, double sec) {
    double per_s = lane_ops / sec;
    printf(", \"%s\": {\"lane_ops_per_s\": %.4g, \"per_clk_per_sm\": %.2f}", name, per_s, per_s / (mhz * 1e6) / sms);
  };
  double it = (double)ITERS * 8 * thr;
  rep("ffma", it, timeit([&] { k_ffma<<<blocks, threads>>>(dout, 0.999f, 0.001f); }));
  rep("ffma2_lanes", 2 * it, timeit([&] { k_ffma2<<<blocks, threads>>>(dout, 0.999f, 0.001f); }));
  rep("ffma2_plus_ffma_lanes", (double)ITERS * 4 * 3 * thr, timeit([&] { k_mix<<<blocks, threads>>>(dout, 0.999f, 0.001f); }));
  rep("fadd2_bcast_ffma2_lanes", (double)ITERS * 4 * 4 * thr, timeit([&] { k_dist<<<blocks, threads>>>(dout, 0.25f); }));
  rep("fadd", it, timeit([&] { k_fadd<<<blocks, threads>>>(dout, 0.001f); }));
  rep("fadd2_lanes", 2 * it, timeit([&] { k_fadd2<<<blocks, threads>>>(dout, 0.001f); }));
  rep("mufu_sqrt", it, timeit([&] { k_mufu<0><<<blocks, threads>>>(dout); }));
  rep("mufu_rsqrt", it, timeit([&] { k_mufu<1><<<blocks, threads>>>(dout); }));
  rep("mufu_ex2", it, timeit([&] { k_mufu<2><<<blocks, threads>>>(dout); }));
  double at = (double)(ITERS / 4) * 8 * thr;
  rep("atoms_lane_private", at, timeit([&] { k_atoms<0><<<blocks, threads, 64 * 32 * 4>>>((unsigned*)dout); }));
  rep("atoms_pure_lane_private", at, timeit([&] { k_atoms_pure<<<blocks, threads, 64 * 32 * 4>>>((unsigned*)dout); }));
  rep("atoms_random_256", at, timeit([&] { k_atoms<1><<<blocks, threads, 64 * 32 * 4>>>((unsigned*)dout); }));
  rep("atoms_same_addr", at, timeit([&] { k_atoms<2><<<blocks, threads, 64 * 32 * 4>>>((unsigned*)dout); }));
  // C4's access pattern: 16384 random bins, R = 2 replicas (128 KB: one 256-thread CTA per SM),
  // R = 1 (64 KB: 1, 2 or 3 CTAs per SM), and 512-thread CTAs sharing the R = 2 copies
  CK(cudaFuncSetAttribute(k_atoms_big<1>, cudaFuncAttributeMaxDynamicSharedMemorySize, 16384 * 2 * 4));
  CK(cudaFuncSetAttribute(k_atoms_big<0>, cudaFuncAttributeMaxDynamicSharedMemorySize, 16384 * 4));
  auto atoms_big = [&](const char* name, int log2r, int cta_per_sm, int thr_per_cta) {
    const double ops = (double)(ITERS / 4) * 8 * sms * cta_per_sm * thr_per_cta;
    const size_t sm_b = (size_t)16384 * 4 << log2r;
    if (log2r == 1) rep(name, ops, timeit([&] { k_atoms_big<1><<<sms * cta_per_sm, thr_per_cta, sm_b>>>((unsigned*)dout, 14); }));
    else rep(name, ops, timeit([&] { k_atoms_big<0><<<sms * cta_per_sm, thr_per_cta, sm_b>>>((unsigned*)dout, 14); }));
  };
  // windows of fewer bins with more replicas (what a spatially sorted tile pair would allow)
  auto atoms_win = [&](const char* name, int log2bins, int log2r, int cta_per_sm, int thr_per_cta) {
    const double ops = (double)(ITERS / 4) * 8 * sms * cta_per_sm * thr_per_cta;
    const size_t sm_b = ((size_t)4 << log2bins) << log2r;
    auto go = [&](auto kern) {
      CK(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm_b));
      rep(name, ops, timeit([&] { kern<<<sms * cta_per_sm, thr_per_cta, sm_b>>>((unsigned*)dout, log2bins); }));
      return 0;
    };
    if (log2r == 2) go(k_atoms_big<2>);
    if (log2r == 3) go(k_atoms_big<3>);
    if (log2r == 4) go(k_atoms_big<4>);
    if (log2r == 5) go(k_atoms_big<5>);
  };
  atoms_win("atoms_random_8k_r4_1x256", 13, 2, 1, 256);
  atoms_win("atoms_random_4k_r8_1x256", 12, 3, 1, 256);
  atoms_win("atoms_random_4k_r8_1x512", 12, 3, 1, 512);
  atoms_win("atoms_random_2k_r16_1x256", 11, 4, 1, 256);
  atoms_win("atoms_random_2k_r16_1x512", 11, 4, 1, 512);
  atoms_win("atoms_random_1k_r32_1x512", 10, 5, 1, 512);
  atoms_win("atoms_random_1k_r32_2x256", 10, 5, 2, 256);
  atoms_big("atoms_random_16k_r2_1x256", 1, 1, 256);
  atoms_big("atoms_random_16k_r2_1x512", 1, 1, 512);
  atoms_big("atoms_random_16k_r2_1x1024", 1, 1, 1024);
  atoms_big("atoms_random_16k_r1_1x256", 0, 1, 256);
  atoms_big("atoms_random_16k_r1_2x256", 0, 2, 256);
  atoms_big("atoms_random_16k_r1_3x256", 0, 3, 256);
  rep("lds128_bcast_instr", (double)ITERS * thr, timeit([&] { k_lds128<<<blocks, threads>>>(dout); }));
  rep("atoms_same_addr_deg2", at, timeit([&] { k_atoms_deg<2><<<blocks, threads, 64 * 32 * 4>>>((unsigned*)dout); }));
  rep("atoms_same_addr_deg4", at, timeit([&] { k_atoms_deg<4><<<blocks, threads, 64 * 32 * 4>>>((unsigned*)dout); }));
  rep("atoms_same_addr_deg8", at, timeit([&] { k_atoms_deg<8><<<blocks, threads, 64 * 32 * 4>>>((unsigned*)dout); }));
  rep("atoms_same_addr_deg16", at, timeit([&] { k_atoms_deg<16><<<blocks, threads, 64 * 32 * 4>>>((unsigned*)dout); }));
  rep("atoms_bank_conflict_deg2", at, timeit([&] { k_atoms_bank<2><<<blocks, threads, 64 * 32 * 4>>>((unsigned*)dout); }));
  rep("atoms_bank_conflict_deg4", at, timeit([&] { k_atoms_bank<4><<<blocks, threads, 64 * 32 * 4>>>((unsigned*)dout); }));
  rep("atoms_bank_conflict_deg8", at, timeit([&] { k_atoms_bank<8><<<blocks, threads, 64 * 32 * 4>>>((unsigned*)dout); }));
  rep("f2i", it, timeit([&] { k_f2i<<<blocks, threads>>>(dout); }));
  rep("shfl_idx_lanes", it, timeit([&] { k_shfl<<<blocks, threads>>>(dout); }));
  size_t bytes = (size_t)8 << 30; float4* big; CK(cudaMalloc(&big, bytes));
  double tw = timeit([&] { k_write<<<sms * 4, 512>>>(big, bytes / 16); });
  printf(", \"hbm_write_stcs_GBps\": %.1f", bytes / tw * 1e-9);
  double tm = timeit([&] { cudaMemsetAsync(big, 0, bytes); });
  printf(", \"hbm_memset_GBps\": %.1f", bytes / tm * 1e-9);
  // re-probe clock after the load
  k_clock<<<sms, 128>>>(dclk, 1 << 22); CK(cudaDeviceSynchronize());
  CK(cudaMemcpy(hclk, dclk, sizeof(hclk), cudaMemcpyDeviceToHost));
  printf(", \"clock_mhz_busy_end\": %.1f}\n", (double)hclk[0] / (double)hclk[1] * 1e3);
  CK(cudaGetLastError());
  return 0;
}
