// tbs_hd2.cuh — high-dimensional Type-III pair matrix on CTA PAIRS (tcgen05 cta_group::2)
// (PAPER.md L330-332 kernel methods over all pairs, Type-III output
// L322-332 / L709-712). Same arithmetic as tbs_hd.cuh (s = |x_i|^2 + |x_j|^2 - 2 x_i . x_j,
// bf16 x bf16 -> fp32), laid out for the L2 bandwidth it needs at large d:
//
//   * the two CTAs of a cluster (two SMs of one TPC) own one 256 x 256 output tile; CTA r
//     loads A rows [256 I + 128 r, +128) and B rows [256 J + 128 r, +128) (its halves of M
//     and N) by TMA into its own shared memory, both completing on the LEADER's mbarrier;
//   * the leader issues tcgen05.mma.cta_group::2 (M = 256, N = 256, K = 16): each SM's
//     tensor core computes its 128 rows x 256 columns from its own A half and BOTH B halves,
//     so every operand byte fetched from L2 serves 256 outputs instead of 128 — 1 B of
//     operand traffic per output per 64-wide k-block instead of 2 (the 128 x 128 one-CTA
//     tile was L2-throughput-bound at d = 512: ~47 B/clk/SM of the ~42 the LTS can deliver);
//   * commits are multicast to both CTAs (operand stage free, accumulator full); both
//     CTAs' epilogues release the accumulator on the leader's barrier;
//   * each CTA's 16 epilogue warps drain its 128 x 256 accumulator in four 64-column quarters
//     through NSTG 32 KB swizzled staging buffers (in turn) and 2-D TMA stores.
#pragma once
#include <cstdint>
#include "tbs_hd.cuh"

namespace tbs {
namespace hd2 {

using hd::kBoxCols;
using hd::kEpiWarps;
using hd::kKBlock;
using hd::kStageBytes;
constexpr int kPair = 256;                         // output tile of a CTA pair (M = N = 256)
constexpr int kHalf = 128;                         // rows (and B rows) per CTA
// Operand ring depth and epilogue staging buffers are template parameters (RING x 32 KB of
// operands + NSTG x 32 KB of staging fit 227 KB for RING + NSTG <= 6): deep rings for large d
// (many k-blocks per tile), more staging buffers — more TMA store groups in flight — when the
// output stream is the bound (small d).
constexpr int kThreads = (kEpiWarps + 2) * 32;     // + a TMA producer warp and an MMA warp
constexpr int kTmemCols = 512;                     // two 256-column fp32 accumulators
constexpr int kNorms = kHalf + kPair;              // per slot: 128 row norms | 256 column norms
constexpr uint32_t kPeerMask = 0xFEFFFFFFu;        // clears the CTA-rank bit of a shared::cluster address
constexpr int kQuarter = 64;                       // columns per epilogue staging step
constexpr int kStageBuf = kHalf * kQuarter * 4;    // 32 KB per staging buffer

template <int RING, int NSTG>
struct Smem {
  static constexpr int OPS = 0;                              // [RING][A | B] x 16 KB
  static constexpr int OPS_STAGE = 2 * kStageBytes;
  static constexpr int STAGE = OPS + RING * OPS_STAGE;       // NSTG x (128 x 64 fp32) staging (2 swizzled boxes each)
  static constexpr int NORMS = STAGE + NSTG * kStageBuf;     // [4 slots][kNorms] fp32
  static constexpr int BARS = NORMS + 4 * kNorms * 4;
  // full[RING] free[RING] acc_full[2] acc_empty[2] nfull[4] nempty[4]
  static constexpr int TMEM = BARS + (2 * RING + 12) * 8;
  static constexpr int BYTES = TMEM + 16;
};

// fp32 accumulate, bf16 A and B, both K-major, N = 256, M = 256 (cta_group::2)
constexpr uint32_t kIdesc = (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(kPair >> 3) << 17) |
                            ((uint32_t)(kPair >> 4) << 24);

__device__ __forceinline__ uint32_t cta_rank() {
  uint32_t r;
  asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
  return r;
}
__device__ __forceinline__ void cluster_sync() {
  asm volatile("barrier.cluster.arrive.release.aligned;\nbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}
// shared::cluster address of the same offset in CTA `rank` of the cluster
__device__ __forceinline__ uint32_t map_rank(uint32_t a, uint32_t rank) {
  uint32_t r;
  asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(r) : "r"(a), "r"(rank));
  return r;
}
// Arrive on an mbarrier of any CTA of the cluster (default .release.cta semantics: the TMEM
// reads it publishes are ordered by tcgen05.fence::before_thread_sync, not by memory fences;
// a .release.cluster arrive costs a MEMBAR.GPU per call, measured as the top epilogue stall).
__device__ __forceinline__ void mbar_arrive_remote(uint32_t cluster_addr) {
  asm volatile("mbarrier.arrive.shared::cluster.b64 _, [%0];" ::"r"(cluster_addr) : "memory");
}
template <int N>
__device__ __forceinline__ void bulk_wait_read() { asm volatile("cp.async.bulk.wait_group.read %0;" ::"n"(N) : "memory"); }
// 32 lanes x 16 consecutive 32-bit TMEM columns -> 16 registers per thread.
__device__ __forceinline__ void tmem_ld16(uint32_t taddr, uint32_t (&v)[16]) {
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
      : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7]), "=r"(v[8]),
        "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]), "=r"(v[14]), "=r"(v[15])
      : "r"(taddr));
  asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
}
// TMA tile load into this CTA's shared memory, completion counted on the LEADER's mbarrier
// (the barrier address with the peer bit cleared).
__device__ __forceinline__ void tma_load_2d_pair(uint32_t dst, const void* tmap, int c0, int c1, uint32_t bar,
                                                 uint64_t policy) {
  asm volatile(
      "cp.async.bulk.tensor.2d.cta_group::2.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint "
      "[%0], [%1, {%2, %3}], [%4], %5;" ::"r"(dst),
      "l"(tmap), "r"(c0), "r"(c1), "r"(bar & kPeerMask), "l"(policy)
      : "memory");
}
// One 64-wide k-block: four K = 16 MMAs on the CTA pair, then the operand stage's commit
// multicast to both CTAs' `free` barriers.
__device__ __forceinline__ void mma_kblock_pair(uint32_t d_tmem, uint64_t a_desc, uint64_t b_desc,
                                                uint32_t accumulate, uint32_t bar) {
  asm volatile(
      "{\n.reg .pred p;\n.reg .b64 a1, a2, a3, b1, b2, b3;\n.reg .b16 m;\n"
      "setp.ne.b32 p, %4, 0;\n"
      "mov.b16 m, 3;\n"
      "add.s64 a1, %1, 2;\nadd.s64 a2, %1, 4;\nadd.s64 a3, %1, 6;\n"
      "add.s64 b1, %2, 2;\nadd.s64 b2, %2, 4;\nadd.s64 b3, %2, 6;\n"
      "tcgen05.mma.cta_group::2.kind::f16 [%0], %1, %2, %3, p;\n"
      "tcgen05.mma.cta_group::2.kind::f16 [%0], a1, b1, %3, 1;\n"
      "tcgen05.mma.cta_group::2.kind::f16 [%0], a2, b2, %3, 1;\n"
      "tcgen05.mma.cta_group::2.kind::f16 [%0], a3, b3, %3, 1;\n"
      "tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%5], m;\n}\n" ::"r"(
          d_tmem),
      "l"(a_desc), "l"(b_desc), "r"(kIdesc), "r"(accumulate), "r"(bar)
      : "memory");
}
__device__ __forceinline__ void commit_pair(uint32_t bar) {
  asm volatile(
      "{\n.reg .b16 m;\nmov.b16 m, 3;\n"
      "tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], m;\n}\n" ::"r"(
          bar)
      : "memory");
}

template <int KTYPE, int RING, int NSTG>
__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(kThreads, 1)
    hd_pair_kernel(const __grid_constant__ CUtensorMap tmap, const __grid_constant__ CUtensorMap tmap_out,
                   int use_tma_store, const float* __restrict__ norms, int n, int kblocks, int I0, int tiles_i,
                   int tiles_j, int rb, int re, float cexp, float* __restrict__ out, int band) {
  using SM = Smem<RING, NSTG>;
  extern __shared__ __align__(1024) unsigned char hd2_smem_raw[];
  unsigned char* sm = reinterpret_cast<unsigned char*>((reinterpret_cast<uintptr_t>(hd2_smem_raw) + 1023) & ~uintptr_t(1023));
  const uint32_t sbase = smem_addr(sm);
  const uint32_t b0 = sbase + SM::BARS;
  auto bar_full = [&](int s) { return b0 + 8 * s; };
  auto bar_free = [&](int s) { return b0 + 8 * (RING + s); };
  auto bar_acc_full = [&](int a) { return b0 + 8 * (2 * RING + a); };
  auto bar_acc_empty = [&](int a) { return b0 + 8 * (2 * RING + 2 + a); };
  auto bar_nfull = [&](int k) { return b0 + 8 * (2 * RING + 4 + k); };
  auto bar_nempty = [&](int k) { return b0 + 8 * (2 * RING + 8 + k); };
  const uint32_t stage = sbase + SM::STAGE;
  const uint32_t snorm = sbase + SM::NORMS;
  uint32_t* tmem_holder = reinterpret_cast<uint32_t*>(sm + SM::TMEM);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const uint32_t rank = cta_rank();
  const int cid = (int)(blockIdx.x >> 1), nclusters = (int)(gridDim.x >> 1);
  const long long ntiles = (long long)tiles_i * tiles_j;

  // Pair tiles: round-robin over clusters in bands of `band` tile rows walked column by column
  // (operand-heavy shapes: the tiles in flight share A bands and B columns in L2), or
  // contiguous row-major ranges (band = 0); both CTAs of a pair walk the same list.
  const bool banded = band > 0;
  const long long c_beg = ntiles * cid / nclusters;
  const long long my_tiles = banded ? (ntiles > cid ? (ntiles - 1 - cid) / nclusters + 1 : 0)
                                    : ntiles * (cid + 1) / nclusters - c_beg;
  auto tile_ij = [&](long long k, int& I, int& J) {
    if (!banded) {
      const long long t = c_beg + k;
      I = I0 + (int)(t / tiles_j);
      J = (int)(t % tiles_j);
      return;
    }
    const long long t = (long long)cid + k * nclusters;
    const long long bi = t / ((long long)band * tiles_j);
    const long long w = t - bi * band * tiles_j;
    const int rows = min(band, tiles_i - (int)bi * band);
    I = I0 + (int)bi * band + (int)(w % rows);
    J = (int)(w / rows);
  };

  if (warp == kEpiWarps) {
    if (lane == 0) {
      for (int k = 0; k < RING; ++k) {
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
  cluster_sync();   // barriers of both CTAs initialised, TMEM allocated, before any remote signal
  // The CTA barrier repeats what the cluster barrier already ordered (the holder written by
  // tcgen05.alloc before any thread reads it) in the form compute-sanitizer's racecheck
  // tracks: it does not model barrier.cluster and reported the holder read as a race (r01).
  __syncthreads();
  hd::tc_fence_after();
  const uint32_t tmem = *tmem_holder;

  if (warp == kEpiWarps) {
    // TMA producer, both CTAs (warp-uniform loop, one elected lane issues).
    const uint64_t keep = hd::policy_evict_last();
    int st = 0;
    uint32_t ph = 0u;
    bool reuse = false;
    for (long long t = 0; t < my_tiles; ++t) {
      int I, J;
      tile_ij(t, I, J);
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
        if (reuse) mbar_wait(bar_free(st), ph ^ 1u);     // the pair's MMAs of the previous pass done
        if (hd::elect_one()) {
          if (rank == 0) mbar_arrive_expect_tx(bar_full(st), (uint32_t)(2 * 2 * kStageBytes));   // both CTAs' bytes
          const uint32_t ops = sbase + SM::OPS + st * SM::OPS_STAGE;
          tma_load_2d_pair(ops, &tmap, kb * kKBlock, I * kPair + rank * kHalf, bar_full(st), keep);
          tma_load_2d_pair(ops + kStageBytes, &tmap, kb * kKBlock, J * kPair + rank * kHalf, bar_full(st), keep);
        }
        __syncwarp();
        if (++st == RING) { st = 0; ph ^= 1u; reuse = true; }
      }
    }
  } else if (warp == kEpiWarps + 1) {
    if (rank == 0) {
      // MMA issuer of the pair (leader CTA only).
      const uint64_t dbase = hd::sw128_desc(sbase + SM::OPS);
      int st = 0;
      uint32_t ph = 0u;
      for (long long t = 0; t < my_tiles; ++t) {
        const int acc = (int)(t & 1);
        const uint32_t d_tmem = tmem + (uint32_t)(acc * kPair);
        if (t >= 2) mbar_wait(bar_acc_empty(acc), (uint32_t)(((t - 2) >> 1) & 1));
        for (int kb = 0; kb < kblocks; ++kb) {
          mbar_wait(bar_full(st), ph);
          hd::tc_fence_after();
          const uint64_t da = dbase + (uint64_t)((st * SM::OPS_STAGE) >> 4);
          if (hd::elect_one()) mma_kblock_pair(d_tmem, da, da + (uint64_t)(kStageBytes >> 4), kb != 0 ? 1u : 0u, bar_free(st));
          __syncwarp();
          if (++st == RING) { st = 0; ph ^= 1u; }
        }
        if (hd::elect_one()) commit_pair(bar_acc_full(acc));
        __syncwarp();
      }
    }
  } else {
    // Epilogue warps: TMEM lane quarter q; each 256-column accumulator row block drains in
    // four 64-column quarters (warp column chunk cq = 16 columns of a quarter) through NSTG
    // 32 KB staging buffers used in turn: quarter k is written while the TMA stores of the
    // NSTG - 1 quarters before it may still be reading theirs, so the store stream (the
    // HBM-bound part) never waits for the compute of the next quarter.
    const int q = warp & 3, cq = warp >> 2;
    const int r = 32 * q + lane;
    const uint64_t stream_out = hd::policy_evict_first();
    const bool storer = threadIdx.x == 0;
    const uint32_t acc_empty_leader[2] = {map_rank(bar_acc_empty(0), 0), map_rank(bar_acc_empty(1), 0)};
    int qs = 0;                                            // staging buffer of the next quarter
    for (long long t = 0; t < my_tiles; ++t) {
      int I, J;
      tile_ij(t, I, J);
      const int acc = (int)(t & 1), ns = (int)(t & 3);
      const int row0 = I * kPair + (int)rank * kHalf;      // first output row of this CTA's half
      const uint32_t nrm = snorm + ns * kNorms * 4;
      mbar_wait(bar_nfull(ns), (uint32_t)((t >> 2) & 1));
      const float ni = hd::ld_shared_f32(nrm + 4 * r);
      mbar_wait(bar_acc_full(acc), (uint32_t)((t >> 1) & 1));
      hd::tc_fence_after();
#pragma unroll 1
      for (int qq = 0; qq < 4; ++qq) {
        const int c16 = qq * kQuarter + 16 * cq;           // this warp's first column in the tile
        float nj[16];
#pragma unroll
        for (int x = 0; x < 16; ++x) nj[x] = hd::ld_shared_f32(nrm + 4 * (kHalf + c16 + x));
        uint32_t v[16];
        tmem_ld16(tmem + ((uint32_t)(32 * q) << 16) + (uint32_t)(acc * kPair + c16), v);
        if (qq == 3) {
          hd::tc_fence_before();
          __syncwarp();
          if (lane == 0) {
            mbar_arrive_remote(acc_empty_leader[acc]);      // accumulator drained (leader's barrier)
            hd::mbar_arrive(bar_nempty(ns));
          }
        }
        float o[16];
#pragma unroll
        for (int x = 0; x < 16; ++x) {
          const float s = fmaf(-2.f, __uint_as_float(v[x]), ni + nj[x]);
          if (KTYPE == 0) o[x] = ex2_approx(cexp * s);
          else if (KTYPE == 1) o[x] = fmaxf(s, 0.f);
          else o[x] = sqrt_approx(fmaxf(s, 0.f));
        }
        const uint32_t buf = stage + (uint32_t)qs * kStageBuf;
        if (++qs == NSTG) qs = 0;
        if (storer) bulk_wait_read<NSTG - 1>();           // stores of quarter k-NSTG have read `buf`
        hd::named_bar(1, kEpiWarps * 32);
#pragma unroll
        for (int x = 0; x < 16; x += 4)
          hd::st_shared_v4(buf + hd::stage_off(r, 16 * cq + x), o[x], o[x + 1], o[x + 2], o[x + 3]);
        hd::fence_async_smem();
        hd::named_bar(1, kEpiWarps * 32);
        const int col0 = J * kPair + qq * kQuarter;
        if (use_tma_store && row0 >= rb) {
          if (storer) {
#pragma unroll
            for (int c = 0; c < kQuarter / kBoxCols; ++c)
              hd::tma_store_2d(&tmap_out, col0 + c * kBoxCols, row0 - rb, buf + c * kHalf * 128, stream_out);
            hd::bulk_commit();
          }
        } else {
          const int jc = col0 + lane;
          for (int rr = warp; rr < kHalf; rr += kEpiWarps) {
            const int gi = row0 + rr;
            if (gi < rb || gi >= re) continue;
            float* dst = out + (size_t)(gi - rb) * (size_t)n;
#pragma unroll
            for (int cc = 0; cc < kQuarter; cc += 32)
              if (jc + cc < n) __stcs(dst + jc + cc, hd::ld_shared_f32(buf + hd::stage_off(rr, lane + cc)));
          }
        }
      }
    }
    if (storer) asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
  }
  hd::tc_fence_before();
  __syncthreads();
  cluster_sync();   // no CTA exits while its peer may still signal it or read its operands
  if (warp == kEpiWarps) {
    hd::tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(kTmemCols) : "memory");
  }
}

}  // namespace hd2
}  // namespace tbs
