// tbs_hd3.cuh — high-dimensional Type-III pair matrix, A-STATIONARY CTA pairs (d <= 512)
// (PAPER.md L330-332 kernel methods over all pairs, Type-III output
// L322-332 / L709-712). Same arithmetic and CTA-pair MMA as tbs_hd2.cuh (s = |x_i|^2 +
// |x_j|^2 - 2 x_i . x_j, bf16 x bf16 -> fp32, tcgen05.mma.cta_group::2, M = N = 256); what
// changes is the operand traffic, which bounds the pair kernel at large d:
//
//   * at d = 512 the hd2 kernel moves 512 KB of operands (A and B halves of a 256 x 256
//     tile) through L2 per 256 KB of output — ~51 GB of L2 traffic per 64K x 64K matrix,
//     at the L2's throughput (~6300 B/clk, B300_MICROARCH);
//   * here a work unit is (tile row I, a range of tile columns): each CTA loads its A half
//     (128 rows x d bf16, all k-blocks, <= 128 KB) ONCE into a resident region and streams
//     only B halves through a 3-stage ring; the A region is refilled when the unit's last
//     MMA has committed (multicast to both CTAs' a_free barriers). Per tile that is 256 KB of
//     operands instead of 512 KB;
//   * the A region takes the space of hd2's second operand half, so the epilogue drains the
//     accumulator in eight 32-column steps through two 16 KB staging buffers.
#pragma once
#include <cstdint>
#include "tbs_hd2.cuh"

namespace tbs {
namespace hd3 {

using hd::kBoxCols;
using hd::kEpiWarps;
using hd::kKBlock;
using hd::kStageBytes;
using hd2::kHalf;
using hd2::kNorms;
using hd2::kPair;
using hd2::kPeerMask;
constexpr int kMaxKBlocks = 8;                     // d <= 512 (A region 8 x 16 KB per CTA)
#ifndef TBS_HD3_RING
#define TBS_HD3_RING 4
#endif
#ifndef TBS_HD3_SBUF
#define TBS_HD3_SBUF 1
#endif
constexpr int kRing = TBS_HD3_RING;                // B ring stages of 16 KB
constexpr int kSBuf = TBS_HD3_SBUF;                // staging buffers of 16 KB
constexpr int kThreads = (kEpiWarps + 2) * 32;
constexpr int kTmemCols = 512;                     // two 256-column fp32 accumulators
constexpr int kStep = 32;                          // accumulator columns per epilogue step
constexpr int kStageBuf = kHalf * kStep * 4;       // 16 KB per staging buffer (one swizzled box)

struct Smem {
  static constexpr int A = 0;                                // [kMaxKBlocks] x 16 KB, resident per unit
  static constexpr int RING = A + kMaxKBlocks * kStageBytes; // [kRing] x 16 KB B halves
  static constexpr int STAGE = RING + kRing * kStageBytes;   // kSBuf x 16 KB staging
  static constexpr int NORMS = STAGE + kSBuf * kStageBuf;    // [4 slots][kNorms] fp32
  static constexpr int BARS = NORMS + 4 * kNorms * 4;
  // full[kRing] free[kRing] acc_full[2] acc_empty[2] nfull[4] nempty[4] a_full a_free
  static constexpr int TMEM = BARS + (2 * kRing + 14) * 8;
  static constexpr int BYTES = TMEM + 16;
};
static_assert(Smem::BYTES + 1024 <= 232448, "A-stationary layout exceeds 227 KB");

// 32 lanes x 8 consecutive 32-bit TMEM columns -> 8 registers per thread.
__device__ __forceinline__ void tmem_ld8(uint32_t taddr, uint32_t (&v)[8]) {
  asm volatile("tcgen05.ld.sync.aligned.32x32b.x8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
               : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7])
               : "r"(taddr));
  asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
}

// Units: (tile row I, column tiles [j0, j1)), `segs` column segments per tile row, dealt
// round-robin over clusters; both CTAs of a pair walk the same list.
__device__ __forceinline__ void unit_of(long long u, int I0, int tiles_j, int segs, int& I, int& j0, int& j1) {
  const int row = (int)(u / segs), sg = (int)(u - (long long)row * segs);
  I = I0 + row;
  j0 = (int)((long long)tiles_j * sg / segs);
  j1 = (int)((long long)tiles_j * (sg + 1) / segs);
}

template <int KTYPE>
__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(kThreads, 1)
    hd_ast_kernel(const __grid_constant__ CUtensorMap tmap, const __grid_constant__ CUtensorMap tmap_out,
                  int use_tma_store, const float* __restrict__ norms, int n, int kblocks, int I0, int tiles_i,
                  int tiles_j, int segs, int rb, int re, float cexp, float* __restrict__ out) {
  extern __shared__ __align__(1024) unsigned char hd3_smem_raw[];
  unsigned char* sm = reinterpret_cast<unsigned char*>((reinterpret_cast<uintptr_t>(hd3_smem_raw) + 1023) & ~uintptr_t(1023));
  const uint32_t sbase = smem_addr(sm);
  const uint32_t b0 = sbase + Smem::BARS;
  auto bar_full = [&](int s) { return b0 + 8 * s; };
  auto bar_free = [&](int s) { return b0 + 8 * (kRing + s); };
  auto bar_acc_full = [&](int a) { return b0 + 8 * (2 * kRing + a); };
  auto bar_acc_empty = [&](int a) { return b0 + 8 * (2 * kRing + 2 + a); };
  auto bar_nfull = [&](int k) { return b0 + 8 * (2 * kRing + 4 + k); };
  auto bar_nempty = [&](int k) { return b0 + 8 * (2 * kRing + 8 + k); };
  const uint32_t bar_afull = b0 + 8 * (2 * kRing + 12), bar_afree = b0 + 8 * (2 * kRing + 13);
  const uint32_t stage = sbase + Smem::STAGE;
  const uint32_t snorm = sbase + Smem::NORMS;
  uint32_t* tmem_holder = reinterpret_cast<uint32_t*>(sm + Smem::TMEM);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const uint32_t rank = hd2::cta_rank();
  const int cid = (int)(blockIdx.x >> 1), nclusters = (int)(gridDim.x >> 1);
  const long long nunits = (long long)tiles_i * segs;
  const long long my_units = nunits > cid ? (nunits - 1 - cid) / nclusters + 1 : 0;

  if (warp == kEpiWarps) {
    if (lane == 0) {
      for (int k = 0; k < kRing; ++k) {
        mbar_init(bar_full(k), 1);
        mbar_init(bar_free(k), 1);
      }
      for (int k = 0; k < 2; ++k) {
        mbar_init(bar_acc_full(k), 1);
        mbar_init(bar_acc_empty(k), 2 * kEpiWarps);   // both CTAs' epilogue warps
      }
      for (int k = 0; k < 4; ++k) {
        mbar_init(bar_nfull(k), 1);
        mbar_init(bar_nempty(k), kEpiWarps);
      }
      mbar_init(bar_afull, 1);
      mbar_init(bar_afree, 1);
      fence_mbar_init();
      asm volatile("prefetch.tensormap [%0];" ::"l"(&tmap) : "memory");
      asm volatile("prefetch.tensormap [%0];" ::"l"(&tmap_out) : "memory");
    }
    __syncwarp();
    asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_addr(tmem_holder)),
                 "r"(kTmemCols)
                 : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;" ::: "memory");
  }
  hd::tc_fence_before();
  hd2::cluster_sync();   // barriers of both CTAs initialised, TMEM allocated, before any remote signal
  hd::tc_fence_after();
  const uint32_t tmem = *tmem_holder;

  if (warp == kEpiWarps) {
    // TMA producer, both CTAs: per unit its A half once, then B halves through the ring.
    const uint64_t keep = hd::policy_evict_last();
    int st = 0;
    uint32_t ph = 0u;
    bool reuse = false;
    long long t = 0;
    for (long long u = 0; u < my_units; ++u) {
      int I, j0, j1;
      unit_of(cid + u * nclusters, I0, tiles_j, segs, I, j0, j1);
      if (u > 0) mbar_wait(bar_afree, (uint32_t)((u - 1) & 1));   // the pair's MMAs on the old A done
      if (hd::elect_one()) {
        if (rank == 0) mbar_arrive_expect_tx(bar_afull, (uint32_t)(2 * kblocks * kStageBytes));   // both CTAs
        for (int kb = 0; kb < kblocks; ++kb)
          hd2::tma_load_2d_pair(sbase + Smem::A + kb * kStageBytes, &tmap, kb * kKBlock, I * kPair + rank * kHalf,
                                bar_afull, keep);
      }
      __syncwarp();
      for (int J = j0; J < j1; ++J, ++t) {
        const int ns = (int)(t & 3);
        if (t >= 4) mbar_wait(bar_nempty(ns), (uint32_t)(((t - 4) >> 2) & 1));
        if (hd::elect_one()) {
          mbar_arrive_expect_tx(bar_nfull(ns), kNorms * 4);
          const uint32_t nd = snorm + ns * kNorms * 4;
          bulk_g2s(nd, norms + (long long)I * kPair + rank * kHalf, kHalf * 4, bar_nfull(ns));
          bulk_g2s(nd + kHalf * 4, norms + (long long)J * kPair, kPair * 4, bar_nfull(ns));
        }
        __syncwarp();
        for (int kb = 0; kb < kblocks; ++kb) {
          if (reuse) mbar_wait(bar_free(st), ph ^ 1u);
          if (hd::elect_one()) {
            if (rank == 0) mbar_arrive_expect_tx(bar_full(st), (uint32_t)(2 * kStageBytes));
            hd2::tma_load_2d_pair(sbase + Smem::RING + st * kStageBytes, &tmap, kb * kKBlock, J * kPair + rank * kHalf,
                                  bar_full(st), keep);
          }
          __syncwarp();
          if (++st == kRing) { st = 0; ph ^= 1u; reuse = true; }
        }
      }
    }
  } else if (warp == kEpiWarps + 1) {
    if (rank == 0) {
      // MMA issuer of the pair (leader CTA only).
      const uint64_t da = hd::sw128_desc(sbase + Smem::A);
      const uint64_t dr = hd::sw128_desc(sbase + Smem::RING);
      int st = 0;
      uint32_t ph = 0u;
      long long t = 0;
      for (long long u = 0; u < my_units; ++u) {
        int I, j0, j1;
        unit_of(cid + u * nclusters, I0, tiles_j, segs, I, j0, j1);
        mbar_wait(bar_afull, (uint32_t)(u & 1));
        hd::tc_fence_after();
        for (int J = j0; J < j1; ++J, ++t) {
          const int acc = (int)(t & 1);
          const uint32_t d_tmem = tmem + (uint32_t)(acc * kPair);
          if (t >= 2) mbar_wait(bar_acc_empty(acc), (uint32_t)(((t - 2) >> 1) & 1));
          hd::tc_fence_after();
          for (int kb = 0; kb < kblocks; ++kb) {
            mbar_wait(bar_full(st), ph);
            hd::tc_fence_after();
            if (hd::elect_one())
              hd2::mma_kblock_pair(d_tmem, da + (uint64_t)((kb * kStageBytes) >> 4),
                                   dr + (uint64_t)((st * kStageBytes) >> 4), kb != 0 ? 1u : 0u, bar_free(st));
            __syncwarp();
            if (++st == kRing) { st = 0; ph ^= 1u; }
          }
          if (hd::elect_one()) hd2::commit_pair(bar_acc_full(acc));
          __syncwarp();
        }
        if (hd::elect_one()) hd2::commit_pair(bar_afree);   // A region free once these MMAs complete
        __syncwarp();
      }
    }
  } else {
    // Epilogue warps: TMEM lane quarter q, 8-column chunk cq of each 32-column step; kSBuf
    // 16 KB staging buffers (with two, step k is written while step k-1's store still reads).
    const int q = warp & 3, cq = warp >> 2;
    const int r = 32 * q + lane;
    const uint64_t stream_out = hd::policy_evict_first();
    const bool storer = threadIdx.x == 0;
    const uint32_t acc_empty_leader[2] = {hd2::map_rank(bar_acc_empty(0), 0), hd2::map_rank(bar_acc_empty(1), 0)};
    long long t = 0;
    int sb = 0;   // staging buffer parity (continues across tiles)
    for (long long u = 0; u < my_units; ++u) {
      int I, j0, j1;
      unit_of(cid + u * nclusters, I0, tiles_j, segs, I, j0, j1);
      const int row0 = I * kPair + (int)rank * kHalf;      // first output row of this CTA's half
      for (int J = j0; J < j1; ++J, ++t) {
        const int acc = (int)(t & 1), ns = (int)(t & 3);
        const uint32_t nrm = snorm + ns * kNorms * 4;
        mbar_wait(bar_nfull(ns), (uint32_t)((t >> 2) & 1));
        const float ni = hd::ld_shared_f32(nrm + 4 * r);
        mbar_wait(bar_acc_full(acc), (uint32_t)((t >> 1) & 1));
        hd::tc_fence_after();
#pragma unroll 1
        for (int qq = 0; qq < kPair / kStep; ++qq) {
          const int c8 = qq * kStep + 8 * cq;                 // this warp's first column in the tile
          float nj[8];
#pragma unroll
          for (int x = 0; x < 8; ++x) nj[x] = hd::ld_shared_f32(nrm + 4 * (kHalf + c8 + x));
          uint32_t v[8];
          tmem_ld8(tmem + ((uint32_t)(32 * q) << 16) + (uint32_t)(acc * kPair + c8), v);
          if (qq == kPair / kStep - 1) {
            hd::tc_fence_before();
            __syncwarp();
            if (lane == 0) {
              hd2::mbar_arrive_remote(acc_empty_leader[acc]);   // accumulator drained (leader's barrier)
              hd::mbar_arrive(bar_nempty(ns));
            }
          }
          float o[8];
#pragma unroll
          for (int x = 0; x < 8; ++x) {
            const float s = fmaf(-2.f, __uint_as_float(v[x]), ni + nj[x]);
            if (KTYPE == 0) o[x] = ex2_approx(cexp * s);
            else if (KTYPE == 1) o[x] = fmaxf(s, 0.f);
            else o[x] = sqrt_approx(fmaxf(s, 0.f));
          }
          const uint32_t buf = stage + (uint32_t)sb * kStageBuf;
          if (++sb == kSBuf) sb = 0;
          if (storer) {                                       // the store that last used `buf` has read it
            if (kSBuf > 1) hd2::bulk_wait_read1();
            else hd::bulk_wait_read0();
          }
          hd::named_bar(1, kEpiWarps * 32);
#pragma unroll
          for (int x = 0; x < 8; x += 4)
            hd::st_shared_v4(buf + hd::stage_off(r, 8 * cq + x), o[x], o[x + 1], o[x + 2], o[x + 3]);
          hd::fence_async_smem();
          hd::named_bar(1, kEpiWarps * 32);
          const int col0 = J * kPair + qq * kStep;
          if (use_tma_store && row0 >= rb) {
            if (storer) {
              hd::tma_store_2d(&tmap_out, col0, row0 - rb, buf, stream_out);
              hd::bulk_commit();
            }
          } else {
            const int jc = col0 + lane;
            for (int rr = warp; rr < kHalf; rr += kEpiWarps) {
              const int gi = row0 + rr;
              if (gi < rb || gi >= re) continue;
              if (jc < n) __stcs(out + (size_t)(gi - rb) * (size_t)n + jc, hd::ld_shared_f32(buf + hd::stage_off(rr, lane)));
            }
          }
        }
      }
    }
    if (storer) asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
  }
  hd::tc_fence_before();
  __syncthreads();
  hd2::cluster_sync();   // no CTA exits while its peer may still signal it or read its operands
  if (warp == kEpiWarps) {
    hd::tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(kTmemCols) : "memory");
  }
}

}  // namespace hd3
}  // namespace tbs
