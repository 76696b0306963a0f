// Exhaustive relative-error bound of sqrt.approx.ftz.f32 on sm_100a, the assumption behind
// the bias-only exact lattice variant (lattice mode): every integer s in
// [1, 2^24) (the whole lattice-mode domain of squared distances) and every fp32 in [1, 4)
// (one full period of the exponent parity). Prints one JSON line.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o sqrt_bound tools/sqrt_bound.cu
#include <cstdio>
#include <cstdint>
#include <cmath>
#include <cstring>
#include <cuda_runtime.h>

#include "../paper_conf_icpp_pitaksirianannt16_b200/csrc/tbs_ptx.cuh"   // tbs::sqrt_sw2

// modes 0, 1: sqrt.approx.ftz.f32 (MUFU); modes 2, 3: tbs::sqrt_sw2 (FMA pipe), same domains
__device__ unsigned long long g_max[4];   // max relative error as ordered double bits

__global__ void k_bound(int mode, uint32_t count) {
  const uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= count) return;
  // mode 0: integers 1 .. 2^24-1; mode 1: fp32 in [1, 4) (bits 0x3f800000 .. 0x407fffff)
  const float x = (mode & 1) == 0 ? (float)(i + 1) : __uint_as_float(0x3f800000u + i);
  float q;
  if (mode < 2) asm("sqrt.approx.ftz.f32 %0, %1;" : "=f"(q) : "f"(x));
  else q = tbs::sqrt_sw2(make_float2(x, x)).x;
  const double t = sqrt((double)x);
  const double e = fabs((double)q - t) / t;
  atomicMax(&g_max[mode], (unsigned long long)__double_as_longlong(e));   // e >= 0: bits are ordered
}

int main() {
  const uint32_t n0 = (1u << 24) - 1, n1 = 0x407fffffu - 0x3f800000u + 1;
  unsigned long long z[4] = {0, 0, 0, 0}, h[4];
  if (cudaMemcpyToSymbol(g_max, z, sizeof(z)) != cudaSuccess) return 1;
  k_bound<<<(n0 + 255) / 256, 256>>>(0, n0);
  k_bound<<<(n1 + 255) / 256, 256>>>(1, n1);
  k_bound<<<(n0 + 255) / 256, 256>>>(2, n0);
  k_bound<<<(n1 + 255) / 256, 256>>>(3, n1);
  if (cudaDeviceSynchronize() != cudaSuccess) return 1;
  cudaMemcpyFromSymbol(h, g_max, sizeof(h));
  double e[4];
  memcpy(e, h, sizeof(e));
  printf("{\"max_rel_err_int\": %.6e, \"log2_int\": %.3f, \"max_rel_err_1_4\": %.6e, \"log2_1_4\": %.3f, "
         "\"sw_max_rel_err_int\": %.6e, \"sw_log2_int\": %.3f, \"sw_max_rel_err_1_4\": %.6e, \"sw_log2_1_4\": %.3f}\n",
         e[0], log2(e[0]), e[1], log2(e[1]), e[2], log2(e[2]), e[3], log2(e[3]));
  return 0;
}
