// tbs_hd.cuh — high-dimensional Type-III pair matrix on the 5th-generation tensor cores
// ("Kernel methods which compute kernel functions
// for all pairs of data in the feature space", Type-III output L322-332 / L709-712).
//
// For d-dimensional bf16 features the pairwise squared distance is
//     s_ij = |x_i|^2 + |x_j|^2 - 2 x_i . x_j,
// and the n x n dot-product matrix is a dense contraction — the one place in this library
// where tensor cores are the right unit (for d >= ~24 FP32 CUDA cores cannot keep up with
// the HBM write rate of the n^2 fp32 output). Per 128 x 128 output tile:
//   * TMA (cp.async.bulk.tensor, SWIZZLE_128B) loads the A rows (tile I) and B rows (tile J),
//     64 bf16 of K per 16 KB box, completion on an mbarrier;
//   * one thread issues tcgen05.mma.kind::f16 (M=128, N=128, K=16 steps, bf16 x bf16 -> fp32)
//     into one of two TMEM accumulators (2 x 128 columns), tcgen05.commit -> mbarriers;
//   * 8 epilogue warps tcgen05.ld the accumulator (32x32b.x32: warp w reads TMEM lanes
//     32 (w % 4).. and columns 64 (w / 4)..), form s from the row / column norms, apply the
//     kernel (ex2 for the Gaussian), stage the tile in shared memory, and write it with
//     coalesced streaming 16-byte stores (each warp row = 512 contiguous bytes).
// A dedicated producer warp overlaps the next tile's loads + MMAs with the epilogue.
#pragma once
#include <cstdint>
#include "tbs_ptx.cuh"

namespace tbs {
namespace hd {

constexpr int kTile = 128;          // M = N = 128
constexpr int kKBlock = 64;         // bf16 per 128-byte swizzle row (one TMA box = 128 x 64)
constexpr int kMaxKBlocks = 2;      // d <= 128
constexpr int kEpiWarps = 8;
constexpr int kThreads = (kEpiWarps + 1) * 32;   // + one producer / MMA warp
constexpr int kStageBytes = kTile * kKBlock * 2; // 16 KB
constexpr int kStageRow = kTile + 4;             // staging row stride (floats): conflict-free
constexpr int kTmemCols = 256;                   // two 128-column fp32 accumulators

struct Smem {
  // offsets from the 1024-aligned dynamic smem base
  static constexpr int A = 0;
  static constexpr int B = A + kMaxKBlocks * kStageBytes;
  static constexpr int STAGE = B + kMaxKBlocks * kStageBytes;
  static constexpr int NORMS = STAGE + kTile * kStageRow * 4;
  static constexpr int BARS = NORMS + kTile * 4;       // full, smem_free, acc_full[2], acc_empty[2]
  static constexpr int TMEM = BARS + 6 * 8;
  static constexpr int BYTES = TMEM + 16;
};

// ---- tcgen05 / TMA wrappers ---------------------------------------------------------
__device__ __forceinline__ void tma_load_2d(uint32_t dst, const void* tmap, int c0, int c1, uint32_t bar) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];" ::"r"(
          dst),
      "l"(tmap), "r"(c0), "r"(c1), "r"(bar)
      : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint32_t bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(bar) : "memory");
}
__device__ __forceinline__ void tc_fence_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void tc_fence_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void tc_commit(uint32_t bar) {
  asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(bar) : "memory");
}
// D[tmem] (+)= A[smem] . B[smem]^T, bf16 inputs, fp32 accumulate (kind::f16).
__device__ __forceinline__ void tc_mma(uint32_t d_tmem, uint64_t a_desc, uint64_t b_desc, uint32_t idesc,
                                       uint32_t accumulate) {
  asm volatile(
      "{\n.reg .pred p;\n"
      "setp.ne.b32 p, %4, 0;\n"
      "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n}\n" ::"r"(d_tmem),
      "l"(a_desc), "l"(b_desc), "r"(idesc), "r"(accumulate)
      : "memory");
}
__device__ __forceinline__ void named_bar(int id, int count) {
  asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(count) : "memory");
}
// 32 lanes x 32 consecutive 32-bit columns of TMEM -> 32 registers per thread.
__device__ __forceinline__ void tmem_ld32(uint32_t taddr, uint32_t (&v)[32]) {
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,"
      "%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
      : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7]), "=r"(v[8]),
        "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]), "=r"(v[14]), "=r"(v[15]), "=r"(v[16]),
        "=r"(v[17]), "=r"(v[18]), "=r"(v[19]), "=r"(v[20]), "=r"(v[21]), "=r"(v[22]), "=r"(v[23]), "=r"(v[24]),
        "=r"(v[25]), "=r"(v[26]), "=r"(v[27]), "=r"(v[28]), "=r"(v[29]), "=r"(v[30]), "=r"(v[31])
      : "r"(taddr));
  asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
}

// Shared-memory matrix descriptor, K-major operand in the canonical SWIZZLE_128B layout
// TMA writes: rows of 128 B, 8-row atoms of 1024 B (stride-dimension byte offset 1024),
// leading-dimension offset unused (1), descriptor version 1, layout type 2 (128B swizzle).
__device__ __forceinline__ uint64_t sw128_desc(uint32_t saddr) {
  return (uint64_t)((saddr >> 4) & 0x3FFFu) | ((uint64_t)1 << 16) | ((uint64_t)(1024 >> 4) << 32) |
         ((uint64_t)1 << 46) | ((uint64_t)2 << 61);
}
// Instruction descriptor: fp32 accumulate, bf16 A and B, both K-major, N = 128, M = 128.
constexpr uint32_t kIdesc = (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(kTile >> 3) << 17) |
                            ((uint32_t)(kTile >> 4) << 24);

// Pad bf16 features [n][d] to [n_pad][dp] (zeros) and compute |x|^2 in fp32 (one warp per row;
// bf16 squares are exact in fp32).
__global__ void hd_prep(const uint16_t* __restrict__ x, int n, int d, int n_pad, int dp, uint16_t* __restrict__ xp,
                        float* __restrict__ norms) {
  const int warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5, lane = threadIdx.x & 31;
  const int nwarps = (gridDim.x * blockDim.x) >> 5;
  for (int r = warp; r < n_pad; r += nwarps) {
    float acc = 0.f;
    for (int c = lane; c < dp; c += 32) {
      const uint16_t h = (r < n && c < d) ? x[(long long)r * d + c] : (uint16_t)0;
      xp[(long long)r * dp + c] = h;
      const float f = __uint_as_float((uint32_t)h << 16);
      acc = fmaf(f, f, acc);
    }
#pragma unroll
    for (int off = 16; off > 0; off >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, off);
    if (lane == 0) norms[r] = acc;
  }
}

template <int KTYPE>
__global__ void __launch_bounds__(kThreads, 1)
    hd_pairmatrix_kernel(const __grid_constant__ CUtensorMap tmap, const float* __restrict__ norms, int n, int kblocks,
                         int I0, int tiles_i, int tiles_j, int rb, int re, float cexp, float* __restrict__ out) {
  extern __shared__ __align__(1024) unsigned char hd_smem_raw[];
  unsigned char* sm = reinterpret_cast<unsigned char*>((reinterpret_cast<uintptr_t>(hd_smem_raw) + 1023) & ~uintptr_t(1023));
  const uint32_t sbase = smem_addr(sm);
  const uint32_t bar_full = sbase + Smem::BARS, bar_free = bar_full + 8;
  const uint32_t bar_acc_full = bar_full + 16, bar_acc_empty = bar_full + 32;   // [2] each
  float* stage = reinterpret_cast<float*>(sm + Smem::STAGE);
  float* snj = reinterpret_cast<float*>(sm + Smem::NORMS);
  uint32_t* tmem_holder = reinterpret_cast<uint32_t*>(sm + Smem::TMEM);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int ntiles = tiles_i * tiles_j;

  if (warp == kEpiWarps) {
    // producer warp: barriers + TMEM allocation (whole warp), then lane 0 drives TMA + MMA
    if (lane == 0) {
      mbar_init(bar_full, 1);
      mbar_init(bar_free, 1);
      mbar_init(bar_acc_full, 1);
      mbar_init(bar_acc_full + 8, 1);
      mbar_init(bar_acc_empty, kEpiWarps);
      mbar_init(bar_acc_empty + 8, kEpiWarps);
      fence_mbar_init();
      asm volatile("prefetch.tensormap [%0];" ::"l"(&tmap) : "memory");
    }
    __syncwarp();
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_addr(tmem_holder)),
                 "r"(kTmemCols)
                 : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tmem_holder;

  if (warp == kEpiWarps) {
    if (lane == 0) {
      int it = 0;
      for (int t = blockIdx.x; t < ntiles; t += gridDim.x, ++it) {
        const int I = I0 + t / tiles_j, J = t % tiles_j, acc = it & 1;
        if (it > 0) mbar_wait(bar_free, (uint32_t)((it - 1) & 1));          // previous MMAs done with smem
        mbar_arrive_expect_tx(bar_full, (uint32_t)(2 * kblocks * kStageBytes));
        for (int kb = 0; kb < kblocks; ++kb) {
          tma_load_2d(sbase + Smem::A + kb * kStageBytes, &tmap, kb * kKBlock, I * kTile, bar_full);
          tma_load_2d(sbase + Smem::B + kb * kStageBytes, &tmap, kb * kKBlock, J * kTile, bar_full);
        }
        mbar_wait(bar_full, (uint32_t)(it & 1));
        if (it >= 2) mbar_wait(bar_acc_empty + 8 * acc, (uint32_t)(((it - 2) >> 1) & 1));   // epilogue drained acc
        tc_fence_after();
        const uint32_t d_tmem = tmem + (uint32_t)(acc * kTile);
        for (int kb = 0; kb < kblocks; ++kb) {
#pragma unroll
          for (int ks = 0; ks < kKBlock / 16; ++ks) {
            const uint64_t da = sw128_desc(sbase + Smem::A + kb * kStageBytes + ks * 32);
            const uint64_t db = sw128_desc(sbase + Smem::B + kb * kStageBytes + ks * 32);
            tc_mma(d_tmem, da, db, kIdesc, (kb | ks) != 0 ? 1u : 0u);
          }
        }
        tc_commit(bar_free);
        tc_commit(bar_acc_full + 8 * acc);
      }
    }
  } else {
    // epilogue warps: TMEM lane quarter q, column half h
    const int q = warp & 3, h = warp >> 2;
    const int et = threadIdx.x;        // 0..255
    int it = 0;
    for (int t = blockIdx.x; t < ntiles; t += gridDim.x, ++it) {
      const int I = I0 + t / tiles_j, J = t % tiles_j, acc = it & 1;
      named_bar(1, kEpiWarps * 32);                       // staging + column norms free
      if (et < kTile) snj[et] = norms[J * kTile + et];
      named_bar(1, kEpiWarps * 32);
      const int r = 32 * q + lane;
      const float ni = norms[I * kTile + r];
      mbar_wait(bar_acc_full + 8 * acc, (uint32_t)((it >> 1) & 1));
      tc_fence_after();
#pragma unroll
      for (int c = 0; c < 2; ++c) {
        const int col0 = 64 * h + 32 * c;
        uint32_t v[32];
        tmem_ld32(tmem + ((uint32_t)(32 * q) << 16) + (uint32_t)(acc * kTile + col0), v);
        float* srow = stage + r * kStageRow + col0;
#pragma unroll
        for (int x = 0; x < 32; x += 4) {
          float o[4];
#pragma unroll
          for (int y = 0; y < 4; ++y) {
            const float s = fmaf(-2.f, __uint_as_float(v[x + y]), ni + snj[col0 + x + y]);
            if (KTYPE == 0) o[y] = ex2_approx(cexp * s);
            else if (KTYPE == 1) o[y] = fmaxf(s, 0.f);
            else o[y] = sqrt_approx(fmaxf(s, 0.f));
          }
          *reinterpret_cast<float4*>(srow + x) = make_float4(o[0], o[1], o[2], o[3]);
        }
      }
      tc_fence_before();
      __syncwarp();
      if (lane == 0) mbar_arrive(bar_acc_empty + 8 * acc);
      named_bar(1, kEpiWarps * 32);                       // tile staged
      // coalesced streaming stores: warp w writes rows w, w+8, ... (512 B per row per warp)
      const int jc = J * kTile + 4 * lane;
      const bool vec = (n & 3) == 0 && jc + 3 < n;
      for (int rr = warp; rr < kTile; rr += kEpiWarps) {
        const int gi = I * kTile + rr;
        if (gi < rb || gi >= re) continue;
        float* dst = out + (size_t)(gi - rb) * (size_t)n + jc;
        const float4 val = *reinterpret_cast<const float4*>(stage + rr * kStageRow + 4 * lane);
        if (vec) {
          st_cs_v4(dst, val.x, val.y, val.z, val.w);
        } else {
          if (jc < n) __stcs(dst, val.x);
          if (jc + 1 < n) __stcs(dst + 1, val.y);
          if (jc + 2 < n) __stcs(dst + 2, val.z);
          if (jc + 3 < n) __stcs(dst + 3, val.w);
        }
      }
    }
  }
  tc_fence_before();
  __syncthreads();
  if (warp == kEpiWarps) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(kTmemCols) : "memory");
  }
}

}  // namespace hd
}  // namespace tbs
