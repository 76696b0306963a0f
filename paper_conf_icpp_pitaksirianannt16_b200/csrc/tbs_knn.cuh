// tbs_knn.cuh — all-point k-nearest neighbours (Type-I, NEXT-2 of SURVEY §8(f)).
//
// PAPER.md L311-313 names "all-point k-nearest neighbors (when k is small)" as a Type-I
// 2-BS: the output of each thread is small enough for registers (L704-709). Reading R5
// (DESIGN.md): per anchor i, the k points j != i of smallest distance in ascending
// (squared distance, j) order; missing entries (n - 1 < k) are (-1, +inf).
//
// Unlike SDH/2PCF the statistic is not symmetric in (i, j) — each anchor owns a list — so the
// schedule is rectangular: CTA (tile, segment) holds KA anchors per thread in registers with
// their K-best lists, and streams the segment's partner chunks through a TMA-staged,
// mbarrier double-buffered shared-memory ring (LDS.128 broadcasts, packed f32x2 distance
// chain as in the pair engine). A candidate is inserted only if strictly better than the
// current K-th entry (one compare per pair; insertions are rare after warm-up). Segments
// write their lists to scratch and a merge kernel combines them in segment (= index) order,
// which keeps the smaller-index-first tie rule exact.
#pragma once
#include <cstdint>
#include "tbs_ptx.cuh"

namespace tbs {
namespace knn {

constexpr int kThreads = 256;
constexpr int kTP = 1024;  // partners per staged chunk

// Insert (v, j) into the ascending list (s, jj) if v < s[K-1]: every entry after the
// insertion point shifts down by one (so equal distances keep their earlier, smaller index
// first); the last entry falls off.
template <int K>
__device__ __forceinline__ void insert(float (&s)[K], int (&jj)[K], float v, int j) {
  bool ins = false;
#pragma unroll
  for (int t = 0; t < K; ++t) {
    const bool sw = ins || (v < s[t]);
    const float ts = s[t];
    const int tj = jj[t];
    s[t] = sw ? v : ts;
    jj[t] = sw ? j : tj;
    v = sw ? ts : v;
    j = sw ? tj : j;
    ins = sw;
  }
}

template <int D>
__device__ __forceinline__ void issue(const float* __restrict__ soa, int n_pad, int c, float* dst, uint32_t bar) {
  mbar_arrive_expect_tx(bar, D * kTP * 4);
#pragma unroll
  for (int d = 0; d < D; ++d)
    bulk_g2s(smem_addr(dst + d * kTP), soa + (long long)d * n_pad + (long long)c * kTP, kTP * 4, bar);
}

// One chunk: every (anchor, partner) pair; SELF masks j == anchor (chunks overlapping the tile).
// Per group of 4 partners: all 4 x KA squared distances first (packed f32x2), then ONE
// predicate "some candidate beats its anchor's current K-th" (a chain of FSETP.OR) and one
// branch; only then the ordered insertions (partner-major, so each anchor sees j ascending).
template <int K, int KA, int D, bool SELF>
__device__ __forceinline__ void chunk(const float* __restrict__ B, int p0, const float2 (&na)[D][KA / 2],
                                      const int (&aidx)[KA], float (&ls)[KA][K], int (&lj)[KA][K]) {
#pragma unroll 1
  for (int p = 0; p < kTP; p += 4) {
    float c4[D][4];
#pragma unroll
    for (int d = 0; d < D; ++d) {
      const float4 v = *reinterpret_cast<const float4*>(B + d * kTP + p);
      c4[d][0] = v.x; c4[d][1] = v.y; c4[d][2] = v.z; c4[d][3] = v.w;
    }
    float2 s[4][KA / 2];
    bool any = false;
#pragma unroll
    for (int q = 0; q < 4; ++q) {
#pragma unroll
      for (int m = 0; m < KA / 2; ++m) {
        float2 dd = __fadd2_rn(na[0][m], make_float2(c4[0][q], c4[0][q]));
        float2 t = __fmul2_rn(dd, dd);
#pragma unroll
        for (int d = 1; d < D; ++d) {
          dd = __fadd2_rn(na[d][m], make_float2(c4[d][q], c4[d][q]));
          t = __ffma2_rn(dd, dd, t);
        }
        if (SELF) {
          const int j = p0 + p + q;
          if (j == aidx[2 * m]) t.x = __int_as_float(0x7f800000);
          if (j == aidx[2 * m + 1]) t.y = __int_as_float(0x7f800000);
        }
        s[q][m] = t;
        any |= (t.x < ls[2 * m][K - 1]) | (t.y < ls[2 * m + 1][K - 1]);
      }
    }
    if (any) {
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        const int j = p0 + p + q;
#pragma unroll
        for (int m = 0; m < KA / 2; ++m) {
          if (s[q][m].x < ls[2 * m][K - 1]) insert<K>(ls[2 * m], lj[2 * m], s[q][m].x, j);
          if (s[q][m].y < ls[2 * m + 1][K - 1]) insert<K>(ls[2 * m + 1], lj[2 * m + 1], s[q][m].y, j);
        }
      }
    }
  }
}

// grid (tiles, S). Tile t: anchors (I0 + t) * TA + k * 256 + tid, k < KA, TA = 256 KA.
// Segment y: partner chunks [y * seg, min((y + 1) * seg, n_chunks)).
// S == 1: writes the first kout entries (idx, sqrt(s)) of rows in [rb, re) directly;
// else the K-list (s, j) to part_s/part_j [y][row - rb][K].
#ifndef TBS_KNN_MINB16
#define TBS_KNN_MINB16 2   // resident CTAs per SM for K <= 16 (A/B knob)
#endif
template <int K, int KA, int D>
__global__ void __launch_bounds__(kThreads, K <= 16 ? TBS_KNN_MINB16 : 1) knn_kernel(const float* __restrict__ soa, int n, int n_pad, int rb, int re,
                                                       int I0, int seg, int n_chunks, int kout,
                                                       float* __restrict__ part_s, int* __restrict__ part_j,
                                                       int* __restrict__ out_idx, float* __restrict__ out_dist) {
  constexpr int TA = kThreads * KA;
  __shared__ __align__(128) float bufs[2][D * kTP];
  __shared__ __align__(8) uint64_t bars[2];
  const int tid = threadIdx.x;
  const int tile = I0 + (int)blockIdx.x;
  const int c0 = (int)blockIdx.y * seg, c1 = min(c0 + seg, n_chunks);
  const uint32_t bar0 = smem_addr(&bars[0]), bar1 = smem_addr(&bars[1]);
  if (tid == 0) {
    mbar_init(bar0, 1);
    mbar_init(bar1, 1);
    fence_mbar_init();
  }
  __syncthreads();
  if (tid == 0 && c0 < c1) issue<D>(soa, n_pad, c0, bufs[0], bar0);

  float2 na[D][KA / 2];
  int aidx[KA];
  float ls[KA][K];
  int lj[KA][K];
#pragma unroll
  for (int k = 0; k < KA; ++k) {
    const int a = tile * TA + k * kThreads + tid;
    aidx[k] = a;
#pragma unroll
    for (int d = 0; d < D; ++d) {
      const float v = -__ldg(soa + (long long)d * n_pad + a);
      if (k & 1) na[d][k >> 1].y = v; else na[d][k >> 1].x = v;
    }
#pragma unroll
    for (int t = 0; t < K; ++t) {
      ls[k][t] = __int_as_float(0x7f800000);
      lj[k][t] = -1;
    }
  }
  const int self_lo = tile * TA / kTP, self_hi = ((tile + 1) * TA - 1) / kTP;  // chunks overlapping the tile
  for (int c = c0, it = 0; c < c1; ++c, ++it) {
    const int s = it & 1;
    if (tid == 0 && c + 1 < c1) issue<D>(soa, n_pad, c + 1, bufs[s ^ 1], s ? bar0 : bar1);
    mbar_wait(s ? bar1 : bar0, (uint32_t)((it >> 1) & 1));
    if (c >= self_lo && c <= self_hi) chunk<K, KA, D, true>(bufs[s], c * kTP, na, aidx, ls, lj);
    else chunk<K, KA, D, false>(bufs[s], c * kTP, na, aidx, ls, lj);
    __syncthreads();  // buffer s is free for the chunk after next
  }
  (void)n;
#pragma unroll
  for (int k = 0; k < KA; ++k) {
    const int a = aidx[k];
    if (a < rb || a >= re) continue;
    if (part_s == nullptr) {
      const size_t o = (size_t)(a - rb) * kout;
#pragma unroll
      for (int t = 0; t < K; ++t)
        if (t < kout) {
          out_idx[o + t] = lj[k][t];
          out_dist[o + t] = sqrtf(ls[k][t]);
        }
    } else {
      const size_t o = ((size_t)blockIdx.y * (size_t)(re - rb) + (size_t)(a - rb)) * K;
#pragma unroll
      for (int t = 0; t < K; ++t) {
        part_s[o + t] = ls[k][t];
        part_j[o + t] = lj[k][t];
      }
    }
  }
}

// Merge the S segment lists of each row, in segment order (increasing partner index).
template <int K>
__global__ void __launch_bounds__(128) knn_merge(const float* __restrict__ part_s, const int* __restrict__ part_j,
                                                 int rows, int S, int kout, int* __restrict__ out_idx,
                                                 float* __restrict__ out_dist) {
  const int r = blockIdx.x * blockDim.x + threadIdx.x;
  if (r >= rows) return;
  float ls[K];
  int lj[K];
#pragma unroll
  for (int t = 0; t < K; ++t) {
    ls[t] = __int_as_float(0x7f800000);
    lj[t] = -1;
  }
  for (int y = 0; y < S; ++y) {
    const size_t o = ((size_t)y * rows + r) * K;
    for (int t = 0; t < K; ++t) {
      const float v = part_s[o + t];
      if (!(v < ls[K - 1])) break;  // the segment's list is ascending
      insert<K>(ls, lj, v, part_j[o + t]);
    }
  }
  const size_t o = (size_t)r * kout;
#pragma unroll
  for (int t = 0; t < K; ++t)
    if (t < kout) {
      out_idx[o + t] = lj[t];
      out_dist[o + t] = sqrtf(ls[t]);
    }
}

}  // namespace knn
}  // namespace tbs
