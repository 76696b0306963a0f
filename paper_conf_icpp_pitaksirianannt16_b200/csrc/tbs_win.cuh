// tbs_win.cuh — spatial order for the WINDOWED large-nb SDH output stage (SURVEY §8(a) a8,
// BASELINE configs[3]: N = 2M, 16384 buckets).
//
// With one shared-memory copy per replica the 16384-bin histogram fits only twice per SM, and a
// warp's 32 increments land in random banks (max-bank-load wavefronts per ATOMS: the measured
// cap of that access pattern). If the points are ordered in space, a work item's
// anchor tile and partner chunk are compact boxes and every pair distance of the item lies in a
// narrow interval [dmin, dmax] of the two boxes: a WINDOW of W consecutive buckets, held with
// 16 replicas (W x 16 words) instead of the whole histogram with 2 — measured 14.7 vs 9.2
// random increments / clk / SM (profiles/r02_peaks.json atoms_random_2k_r16 vs 16k_r2). Items
// whose interval is wider than W run as several window segments with an in-range check.
//
// The order: a counting sort of the points by the Morton code of their cell on a 2^g grid over
// the loader's bounding box (points of one cell in arbitrary order). The SDH is a function of
// the point SET, so the order never changes the histogram; it is used only for full-range calls
// (a row range names anchors by the caller's indices).
#pragma once
#include <cstdint>
#include "tbs_kernels.cuh"

namespace tbs {
namespace win {

// 10 bits -> every third bit (Morton interleave of 3 coordinates)
__device__ __forceinline__ uint32_t spread3(uint32_t v) {
  v &= 0x3ffu;
  v = (v | (v << 16)) & 0x030000FFu;
  v = (v | (v << 8)) & 0x0300F00Fu;
  v = (v | (v << 4)) & 0x030C30C3u;
  v = (v | (v << 2)) & 0x09249249u;
  return v;
}

// Cell (Morton code on a 2^g grid over the box recorded by the loader) of every point; counts.
__global__ void cell_count(const float* __restrict__ soa, int n, int n_pad, const uint32_t* __restrict__ bbox, int g,
                           uint32_t* __restrict__ cell, uint32_t* __restrict__ count) {
  float lo[3], sc[3];
  const float G = (float)(1 << g);
#pragma unroll
  for (int c = 0; c < 3; ++c) {
    lo[c] = ord2f(~bbox[c]);
    const float ext = ord2f(bbox[3 + c]) - lo[c];
    sc[c] = ext > 0.f ? G / ext : 0.f;
  }
  const int top = (1 << g) - 1;
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) {
    uint32_t code = 0;
#pragma unroll
    for (int c = 0; c < 3; ++c) {
      const float t = (soa[(long long)c * n_pad + i] - lo[c]) * sc[c];
      const int q = t >= 0.f ? min((int)t, top) : 0;   // (NaN -> 0: the order is only a heuristic)
      code |= spread3((uint32_t)q) << c;
    }
    cell[i] = code;
    atomicAdd(count + code, 1u);
  }
}

// In-place exclusive prefix sum of m counts: one CTA of 1024 threads, each a contiguous run.
__global__ void __launch_bounds__(1024) scan_exclusive(uint32_t* __restrict__ a, int m) {
  __shared__ uint32_t part[1024];
  const int t = threadIdx.x;
  const int per = (m + 1023) / 1024, b = t * per, e = min(b + per, m);
  uint32_t s = 0;
  for (int i = b; i < e; ++i) s += a[i];
  part[t] = s;
  __syncthreads();
  for (int off = 1; off < 1024; off <<= 1) {   // Hillis-Steele inclusive scan of the run sums
    const uint32_t v = t >= off ? part[t - off] : 0u;
    __syncthreads();
    part[t] += v;
    __syncthreads();
  }
  uint32_t run = part[t] - s;                   // exclusive start of this thread's run
  for (int i = b; i < e; ++i) {
    const uint32_t v = a[i];
    a[i] = run;
    run += v;
  }
}

// Scatter point i to the next free slot of its cell (offs: the exclusive scan, advanced).
__global__ void scatter_cells(const float* __restrict__ soa, int n, int n_pad, const uint32_t* __restrict__ cell,
                              uint32_t* __restrict__ offs, float* __restrict__ out) {
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) {
    const uint32_t p = atomicAdd(offs + cell[i], 1u);
#pragma unroll
    for (int c = 0; c < 3; ++c) out[(long long)c * n_pad + p] = soa[(long long)c * n_pad + i];
  }
}

// Box (lo[3], hi[3]) of the valid points of every TP-point chunk of the ordered SoA; a chunk
// with no valid point gets lo = +inf, hi = -inf. One CTA (256 threads) per chunk.
__global__ void __launch_bounds__(256) chunk_boxes(const float* __restrict__ soa, int n, int n_pad, int tp,
                                                   float* __restrict__ boxes) {
  __shared__ float red[6][8];
  const int ch = blockIdx.x, t = threadIdx.x;
  float lo[3], hi[3];
#pragma unroll
  for (int c = 0; c < 3; ++c) {
    lo[c] = __int_as_float(0x7f800000);
    hi[c] = -__int_as_float(0x7f800000);
  }
  for (int k = t; k < tp; k += 256) {
    const long long i = (long long)ch * tp + k;
    if (i < n) {
#pragma unroll
      for (int c = 0; c < 3; ++c) {
        const float v = soa[(long long)c * n_pad + i];
        lo[c] = fminf(lo[c], v);
        hi[c] = fmaxf(hi[c], v);
      }
    }
  }
#pragma unroll
  for (int c = 0; c < 3; ++c) {
#pragma unroll
    for (int off = 16; off > 0; off >>= 1) {
      lo[c] = fminf(lo[c], __shfl_xor_sync(0xffffffffu, lo[c], off));
      hi[c] = fmaxf(hi[c], __shfl_xor_sync(0xffffffffu, hi[c], off));
    }
  }
  if ((t & 31) == 0) {
#pragma unroll
    for (int c = 0; c < 3; ++c) {
      red[c][t >> 5] = lo[c];
      red[3 + c][t >> 5] = hi[c];
    }
  }
  __syncthreads();
  if (t < 6) {
    float v = red[t][0];
    for (int w = 1; w < 8; ++w) v = t < 3 ? fminf(v, red[t][w]) : fmaxf(v, red[t][w]);
    boxes[(long long)ch * 6 + t] = v;
  }
}

}  // namespace win
}  // namespace tbs
