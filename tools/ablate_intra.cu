// Fig. 7 ablation on B200 (§IV-E1 "load balancing" of the intra-block
// pairs, Alg. 2 l.9-12 / Alg. 3 l.10-14): the time of the INTRA-block (diagonal) part of the
// SDH alone, under three schedules of the i<j pairs inside a block of B points (one point per
// thread, the paper's layout), each feeding the same output stage as the product kernel
// (32 lane-private u32 histogram copies, sqrt.approx + round-down bucket, red.shared.add):
//   naive    thread t pairs with j = t+1 .. B-1          (unequal trip counts: divergence)
//   masked   every thread walks j = 0 .. B-1 with the     (this repo's diagonal items: equal
//            predicate j > t, partner j broadcast         trip counts, half the slots masked)
//   lb       thread t pairs with (t + j) mod B,           (the paper's load-balanced schedule:
//            j = 1 .. B/2, the last step for t < B/2 only equal trip counts, per-lane partners)
// Every schedule counts each pair once and computes the same fp32 distance ((a-p)^2 = (p-a)^2
// exactly), so the histograms must be identical: checked. Prints one JSON line per (B, schedule).
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o ablate_intra tools/ablate_intra.cu
#include <cstdint>
#include <cstdio>
#include <cstring>
#include <vector>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e_ = (x); if (e_ != cudaSuccess) { \
  fprintf(stderr, "%s:%d %s\n", __FILE__, __LINE__, cudaGetErrorString(e_)); return 1; } } while (0)

constexpr int NB = 256;                 // buckets (C2/C6's 256)
constexpr uint32_t kMagic = 0x4B000000u;

__device__ __forceinline__ float sqrt_approx(float x) {
  float r;
  asm("sqrt.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(x));
  return r;
}
__device__ __forceinline__ void inc(uint32_t* h, float s, float inv_w, int lane) {
  const float y = __fmaf_rd(sqrt_approx(s), inv_w, 8388608.0f);
  const uint32_t k = min(__float_as_uint(y) - kMagic, (uint32_t)(NB - 1));
  atomicAdd(h + k * 32 + lane, 1u);
}

template <int MODE>
__global__ void intra(const float* __restrict__ pts, int B, float inv_w, unsigned long long* __restrict__ hist, int reps) {
  extern __shared__ float sm[];
  float* sx = sm;
  float* sy = sm + B;
  float* sz = sm + 2 * B;
  uint32_t* h = reinterpret_cast<uint32_t*>(sm + 3 * B);
  const int t = threadIdx.x, lane = t & 31;
  for (int i = t; i < NB * 32; i += B) h[i] = 0u;
  const long long base = (long long)blockIdx.x * B;
  const float ax = pts[3 * (base + t)], ay = pts[3 * (base + t) + 1], az = pts[3 * (base + t) + 2];
  sx[t] = ax; sy[t] = ay; sz[t] = az;
  __syncthreads();
  for (int r = 0; r < reps; ++r) {
    if (MODE == 0) {
      for (int j = t + 1; j < B; ++j) {
        const float dx = sx[j] - ax, dy = sy[j] - ay, dz = sz[j] - az;
        inc(h, fmaf(dz, dz, fmaf(dy, dy, dx * dx)), inv_w, lane);
      }
    } else if (MODE == 1) {
      for (int j = 0; j < B; ++j) {
        const float dx = sx[j] - ax, dy = sy[j] - ay, dz = sz[j] - az;
        const float s = fmaf(dz, dz, fmaf(dy, dy, dx * dx));
        if (j > t) inc(h, s, inv_w, lane);
      }
    } else {
      for (int j = 1; j < B / 2; ++j) {
        const int q = (t + j) & (B - 1);
        const float dx = sx[q] - ax, dy = sy[q] - ay, dz = sz[q] - az;
        inc(h, fmaf(dz, dz, fmaf(dy, dy, dx * dx)), inv_w, lane);
      }
      if (t < B / 2) {                       // the last step: only the lower half (L1094-1097)
        const int q = t + B / 2;
        const float dx = sx[q] - ax, dy = sy[q] - ay, dz = sz[q] - az;
        inc(h, fmaf(dz, dz, fmaf(dy, dy, dx * dx)), inv_w, lane);
      }
    }
  }
  __syncthreads();
  for (int k = t; k < NB; k += B) {
    unsigned long long v = 0;
    for (int l = 0; l < 32; ++l) v += h[k * 32 + l];
    if (v) atomicAdd(hist + k, v);
  }
}

static uint64_t splitmix(uint64_t& x) {
  uint64_t z = (x += 0x9E3779B97F4A7C15ull);
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

int main() {
  cudaDeviceProp prop;
  CK(cudaGetDeviceProperties(&prop, 0));
  const int sms = prop.multiProcessorCount;
  const char* names[3] = {"naive", "masked", "lb"};
  for (int B : {256, 1024}) {
    const int blocks = sms * (B == 256 ? 32 : 8);       // many waves of intra-block tiles
    const int reps = B == 256 ? 16 : 4;
    const long long n = (long long)blocks * B;
    std::vector<float> hp(3 * n);
    uint64_t st = 7;
    for (auto& v : hp) v = (float)(splitmix(st) >> 40) * (1.0f / 16777216.0f);
    float* dp;
    unsigned long long* dh;
    CK(cudaMalloc(&dp, hp.size() * 4));
    CK(cudaMalloc(&dh, NB * 8));
    CK(cudaMemcpy(dp, hp.data(), hp.size() * 4, cudaMemcpyHostToDevice));
    const float inv_w = (float)(256.0 / 1.7320508075688772);
    const size_t smem = 3 * B * 4 + NB * 32 * 4;
    std::vector<unsigned long long> ref(NB), cur(NB);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    for (int mode = 0; mode < 3; ++mode) {
      auto launch = [&](int rp) {
        if (mode == 0) intra<0><<<blocks, B, smem>>>(dp, B, inv_w, dh, rp);
        if (mode == 1) intra<1><<<blocks, B, smem>>>(dp, B, inv_w, dh, rp);
        if (mode == 2) intra<2><<<blocks, B, smem>>>(dp, B, inv_w, dh, rp);
      };
      CK(cudaFuncSetAttribute(intra<0>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
      CK(cudaFuncSetAttribute(intra<1>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
      CK(cudaFuncSetAttribute(intra<2>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
      CK(cudaMemset(dh, 0, NB * 8));
      launch(1);                                        // correctness: one rep
      CK(cudaDeviceSynchronize());
      CK(cudaMemcpy(cur.data(), dh, NB * 8, cudaMemcpyDeviceToHost));
      unsigned long long mass = 0;
      for (auto v : cur) mass += v;
      const bool mass_ok = mass == (unsigned long long)blocks * B * (B - 1) / 2;
      if (mode == 0) ref = cur;
      const bool same = cur == ref;
      launch(reps);                                     // warm
      CK(cudaDeviceSynchronize());
      float best = 1e30f;
      for (int it = 0; it < 5; ++it) {
        cudaEventRecord(e0);
        launch(reps);
        cudaEventRecord(e1);
        CK(cudaEventSynchronize(e1));
        float ms;
        cudaEventElapsedTime(&ms, e0, e1);
        if (ms < best) best = ms;
      }
      const double pairs = (double)blocks * reps * B * (B - 1) / 2.0;
      printf("{\"ablation\": \"intra_block_schedule\", \"paper\": \"Fig. 7 (L1076-1107)\", \"B\": %d, \"schedule\": \"%s\", "
             "\"blocks\": %d, \"reps\": %d, \"ms\": %.4f, \"gpairs_s\": %.2f, \"mass_ok\": %s, \"hist_equal_naive\": %s}\n",
             B, names[mode], blocks, reps, best, pairs / best / 1e6, mass_ok ? "true" : "false", same ? "true" : "false");
    }
    cudaFree(dp);
    cudaFree(dh);
  }
  return 0;
}
