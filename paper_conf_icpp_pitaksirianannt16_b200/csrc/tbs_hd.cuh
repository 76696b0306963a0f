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
//   * 16 epilogue warps tcgen05.ld the accumulator (32x32b.x32: warp w reads TMEM lanes
//     32 (w % 4).. and columns 32 (w / 4)..), form s from the row / column norms (bulk-copied
//     into shared memory by the producer beside the operands), apply the kernel (ex2 for the
//     Gaussian), stage the tile in shared memory, and write it with coalesced streaming
//     16-byte stores (each warp row = 512 contiguous bytes).
// A TMA producer warp and an MMA-issuer warp overlap the next tile's loads + MMAs with the epilogue.
#pragma once
#include <cstdint>
#include "tbs_ptx.cuh"

namespace tbs {
namespace hd {

constexpr int kTile = 128;          // M = N = 128
constexpr int kKBlock = 64;         // bf16 per 128-byte swizzle row (one TMA box = 128 x 64)
constexpr int kRing = 4;            // operand ring: 4 stages of (A, B) k-blocks = 128 KB
constexpr int kMaxD = 1024;         // feature dimension limit (k-blocks stream through the ring)
constexpr int kEpiWarps = 16;                    // 4 TMEM lane quarters x 4 column chunks of 32
constexpr int kThreads = (kEpiWarps + 2) * 32;   // + a TMA producer warp and an MMA warp
constexpr int kStageBytes = kTile * kKBlock * 2; // 16 KB
constexpr int kBoxCols = 32;                     // output TMA box: 128 rows x 32 fp32 (128 B, SWIZZLE_128B)
constexpr int kTmemCols = 256;                   // two 128-column fp32 accumulators
constexpr int kBand = 16;                        // tile rows per raster band

struct Smem {
  // offsets from the 1024-aligned dynamic smem base
  static constexpr int OPS = 0;                                  // [kRing][A | B] x 16 KB
  static constexpr int OPS_STAGE = 2 * kStageBytes;
  static constexpr int STAGE = OPS + kRing * OPS_STAGE;          // output staging tile (4 swizzled boxes)
  static constexpr int NORMS = STAGE + kTile * kTile * 4;        // [4 slots][rows I | cols J] x 128 fp32
  static constexpr int BARS = NORMS + 4 * 2 * kTile * 4;
  // barriers: full[kRing] free[kRing] acc_full[2] acc_empty[2] nfull[4] nempty[4]
  static constexpr int TMEM = BARS + (2 * kRing + 12) * 8;
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
// One k-block of 64 = four K=16 MMAs (descriptors advance 32 B = 2 units per K step) and the
// commit of the operand stage, in ONE asm block issued by one elected lane of a warp-uniform
// loop: per-instruction elect/uniform-register overhead would otherwise make the issuing
// thread slower than the tensor pipe (measured: ~115 SASS instructions per k-block).
__device__ __forceinline__ void tc_mma_kblock(uint32_t d_tmem, uint64_t a_desc, uint64_t b_desc, uint32_t idesc,
                                              uint32_t accumulate, uint32_t bar) {
  asm volatile(
      "{\n.reg .pred p;\n.reg .b64 a1, a2, a3, b1, b2, b3;\n"
      "setp.ne.b32 p, %4, 0;\n"
      "add.s64 a1, %1, 2;\nadd.s64 a2, %1, 4;\nadd.s64 a3, %1, 6;\n"
      "add.s64 b1, %2, 2;\nadd.s64 b2, %2, 4;\nadd.s64 b3, %2, 6;\n"
      "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n"
      "tcgen05.mma.cta_group::1.kind::f16 [%0], a1, b1, %3, 1;\n"
      "tcgen05.mma.cta_group::1.kind::f16 [%0], a2, b2, %3, 1;\n"
      "tcgen05.mma.cta_group::1.kind::f16 [%0], a3, b3, %3, 1;\n"
      "tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%5];\n}\n" ::"r"(d_tmem),
      "l"(a_desc), "l"(b_desc), "r"(idesc), "r"(accumulate), "r"(bar)
      : "memory");
}
__device__ __forceinline__ bool elect_one() {
  uint32_t e;
  asm volatile("{\n.reg .pred p;\nelect.sync _|p, 0xffffffff;\nselp.u32 %0, 1, 0, p;\n}\n" : "=r"(e));
  return e != 0u;
}
// TMA 1-D bulk store shared -> global (bulk async-group completion), used to drain the
// staged output tile without occupying the warps (SASS: UBLKCP).
__device__ __forceinline__ void bulk_s2g(void* dst, uint32_t src, uint32_t bytes) {
  asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(dst), "r"(src), "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void bulk_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
__device__ __forceinline__ void bulk_wait_read0() { asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory"); }
__device__ __forceinline__ void fence_async_smem() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }
// 2-D TMA tensor store shared -> global with an L2 eviction-priority hint.
__device__ __forceinline__ void tma_store_2d(const void* tmap, int c0, int c1, uint32_t src, uint64_t policy) {
  asm volatile("cp.async.bulk.tensor.2d.global.shared::cta.bulk_group.L2::cache_hint [%0, {%1, %2}], [%3], %4;" ::"l"(
                   tmap),
               "r"(c0), "r"(c1), "r"(src), "l"(policy)
               : "memory");
}
__device__ __forceinline__ void tma_load_2d_hint(uint32_t dst, const void* tmap, int c0, int c1, uint32_t bar,
                                                 uint64_t policy) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1, {%2, %3}], "
      "[%4], %5;" ::"r"(dst),
      "l"(tmap), "r"(c0), "r"(c1), "r"(bar), "l"(policy)
      : "memory");
}
__device__ __forceinline__ uint64_t policy_evict_first() {
  uint64_t p;
  asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
  return p;
}
__device__ __forceinline__ uint64_t policy_evict_last() {
  uint64_t p;
  asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
  return p;
}
__device__ __forceinline__ void st_shared_v4(uint32_t a, float x, float y, float z, float w) {
  asm volatile("st.shared.v4.f32 [%0], {%1, %2, %3, %4};" ::"r"(a), "f"(x), "f"(y), "f"(z), "f"(w) : "memory");
}
__device__ __forceinline__ float ld_shared_f32(uint32_t a) {
  float v;
  asm volatile("ld.shared.f32 %0, [%1];" : "=f"(v) : "r"(a) : "memory");
  return v;
}
// Byte offset of output element (row, col) in the staging tile: 4 boxes of 128 rows x 32 fp32
// (one per 32-column chunk), each row 128 B with the TMA SWIZZLE_128B pattern (16-byte chunk
// index XOR row % 8) — conflict-free for one-row-per-lane writes, and the layout a 2-D TMA
// store of a [128 x 32] box with SWIZZLE_128B reads.
__device__ __forceinline__ uint32_t stage_off(int row, int col) {
  return (uint32_t)((col >> 5) * (kTile * 128) + row * 128 + ((((col & 31) >> 2) ^ (row & 7)) << 4) + (col & 3) * 4);
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
    hd_pairmatrix_kernel(const __grid_constant__ CUtensorMap tmap, const __grid_constant__ CUtensorMap tmap_out,
                         int use_tma_store, const float* __restrict__ norms, int n, int kblocks, int I0, int tiles_i,
                         int tiles_j, int rb, int re, float cexp, float* __restrict__ out) {
  extern __shared__ __align__(1024) unsigned char hd_smem_raw[];
  unsigned char* sm = reinterpret_cast<unsigned char*>((reinterpret_cast<uintptr_t>(hd_smem_raw) + 1023) & ~uintptr_t(1023));
  const uint32_t sbase = smem_addr(sm);
  const uint32_t b0 = sbase + Smem::BARS;
  auto bar_full = [&](int s) { return b0 + 8 * s; };
  auto bar_free = [&](int s) { return b0 + 8 * (kRing + s); };
  auto bar_acc_full = [&](int a) { return b0 + 8 * (2 * kRing + a); };
  auto bar_acc_empty = [&](int a) { return b0 + 8 * (2 * kRing + 2 + a); };
  auto bar_nfull = [&](int k) { return b0 + 8 * (2 * kRing + 4 + k); };
  auto bar_nempty = [&](int k) { return b0 + 8 * (2 * kRing + 8 + k); };
  const uint32_t stage = sbase + Smem::STAGE;
  const uint32_t snorm = sbase + Smem::NORMS;                                   // [slot][2][128] fp32
  uint32_t* tmem_holder = reinterpret_cast<uint32_t*>(sm + Smem::TMEM);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const long long ntiles = (long long)tiles_i * tiles_j;
  // Operand-heavy shapes (kblocks > 2): tiles are dealt round-robin (CTA b takes tiles b,
  // b + grid, ...), so the grid works on ~grid consecutive tiles at a time, and consecutive
  // tiles follow a grouped raster: bands of kBand tile rows walked column by column. The tiles
  // in flight then share a few B column blocks and one A band (L2 hits; DRAM operand reads
  // 7.2 GB -> 2.1 GB at 64K x 512). Output-bound shapes (small d) keep a contiguous row-major
  // range per CTA (each CTA streams whole output rows: measured faster at d = 64).
  const bool banded = kblocks > 2;
  const long long c_beg = ntiles * blockIdx.x / gridDim.x;
  const long long my_tiles = banded ? (ntiles > blockIdx.x ? (ntiles - 1 - blockIdx.x) / gridDim.x + 1 : 0)
                                    : ntiles * (blockIdx.x + 1) / gridDim.x - c_beg;
  auto tile_ij = [&](long long k, int& I, int& J) {
    if (!banded) {
      const long long t = c_beg + k;
      I = I0 + (int)(t / tiles_j);
      J = (int)(t % tiles_j);
      return;
    }
    const long long t = (long long)blockIdx.x + k * gridDim.x;
    const long long band = t / ((long long)kBand * tiles_j);
    const long long w = t - band * kBand * tiles_j;
    const int rows = min(kBand, tiles_i - (int)band * kBand);
    I = I0 + (int)band * kBand + (int)(w % rows);
    J = (int)(w / rows);
  };

  if (warp == kEpiWarps) {
    if (lane == 0) {
      for (int k = 0; k < kRing; ++k) {
        mbar_init(bar_full(k), 1);
        mbar_init(bar_free(k), 1);
      }
      for (int k = 0; k < 2; ++k) {
        mbar_init(bar_acc_full(k), 1);
        mbar_init(bar_acc_empty(k), kEpiWarps);
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
    // TMA producer (warp-uniform loop, one elected lane issues). Operand k-blocks of
    // consecutive tiles stream through a kRing-deep ring (stage st, pass parity ph kept
    // incrementally: no divisions on this critical path); a tile's norms go into a 4-slot
    // ring with its first k-block. Every wait is on the completion right after the last one
    // consumed for that barrier.
    const uint64_t keep = policy_evict_last();
    int st = 0;
    uint32_t ph = 0u;
    bool reuse = false;                                    // ring wrapped at least once
    for (long long t = 0; t < my_tiles; ++t) {
      int I, J;
      tile_ij(t, I, J);
      const int ns = (int)(t & 3);
      if (t >= 4) mbar_wait(bar_nempty(ns), (uint32_t)(((t - 4) >> 2) & 1));        // epilogue of t-4 read slot
      if (elect_one()) {
        mbar_arrive_expect_tx(bar_nfull(ns), 2 * kTile * 4);
        const uint32_t nd = sbase + Smem::NORMS + ns * 2 * kTile * 4;
        bulk_g2s(nd, norms + I * kTile, kTile * 4, bar_nfull(ns));
        bulk_g2s(nd + kTile * 4, norms + J * kTile, kTile * 4, bar_nfull(ns));
      }
      __syncwarp();
      for (int kb = 0; kb < kblocks; ++kb) {
        if (reuse) mbar_wait(bar_free(st), ph ^ 1u);       // MMAs of the previous pass over st done
        if (elect_one()) {
          mbar_arrive_expect_tx(bar_full(st), (uint32_t)(2 * kStageBytes));
          const uint32_t ops = sbase + Smem::OPS + st * Smem::OPS_STAGE;
          // features stay L2-resident (evict_last) under the output stream
          tma_load_2d_hint(ops, &tmap, kb * kKBlock, I * kTile, bar_full(st), keep);
          tma_load_2d_hint(ops + kStageBytes, &tmap, kb * kKBlock, J * kTile, bar_full(st), keep);
        }
        __syncwarp();
        if (++st == kRing) { st = 0; ph ^= 1u; reuse = true; }
      }
    }
  } else if (warp == kEpiWarps + 1) {
    // MMA issuer (warp-uniform loop, one elected lane issues): per k-block wait for its
    // operands, four K=16 MMAs into the tile's accumulator and the commit of the stage back
    // to the producer; per tile, commit the accumulator to the epilogue.
    const uint64_t dbase = sw128_desc(sbase + Smem::OPS);     // + (byte offset >> 4) per operand
    int st = 0;
    uint32_t ph = 0u;
    for (long long t = 0; t < my_tiles; ++t) {
      const int acc = (int)(t & 1);
      const uint32_t d_tmem = tmem + (uint32_t)(acc * kTile);
      if (t >= 2) mbar_wait(bar_acc_empty(acc), (uint32_t)(((t - 2) >> 1) & 1));    // acc drained
      for (int kb = 0; kb < kblocks; ++kb) {
        mbar_wait(bar_full(st), ph);
        tc_fence_after();
        const uint64_t da = dbase + (uint64_t)((st * Smem::OPS_STAGE) >> 4);
        if (elect_one()) tc_mma_kblock(d_tmem, da, da + (uint64_t)(kStageBytes >> 4), kIdesc, kb != 0 ? 1u : 0u, bar_free(st));
        __syncwarp();
        if (++st == kRing) { st = 0; ph ^= 1u; }
      }
      if (elect_one()) tc_commit(bar_acc_full(acc));
      __syncwarp();
    }
  } else {
    // epilogue warps: TMEM lane quarter q, 32-column chunk cq
    const int q = warp & 3, cq = warp >> 2;
    const int r = 32 * q + lane;
    const uint64_t stream_out = policy_evict_first();
    const bool storer = threadIdx.x == 0;                 // issues the tile's four TMA stores
    int it = 0;
    for (long long t = 0; t < my_tiles; ++t, ++it) {
      int I, J;
      tile_ij(t, I, J);
      const int acc = it & 1, ns = it & 3;
      const uint32_t nrm = snorm + ns * 2 * kTile * 4;
      mbar_wait(bar_nfull(ns), (uint32_t)((it >> 2) & 1));
      const float ni = ld_shared_f32(nrm + 4 * r);
      float nj[32];
#pragma unroll
      for (int x = 0; x < 32; ++x) nj[x] = ld_shared_f32(nrm + 4 * (kTile + 32 * cq + x));
      __syncwarp();
      if (lane == 0) mbar_arrive(bar_nempty(ns));
      mbar_wait(bar_acc_full(acc), (uint32_t)((it >> 1) & 1));
      tc_fence_after();
      uint32_t v[32];
      tmem_ld32(tmem + ((uint32_t)(32 * q) << 16) + (uint32_t)(acc * kTile + 32 * cq), v);
      tc_fence_before();
      __syncwarp();
      if (lane == 0) mbar_arrive(bar_acc_empty(acc));
      float o[32];
#pragma unroll
      for (int x = 0; x < 32; ++x) {
        const float s = fmaf(-2.f, __uint_as_float(v[x]), ni + nj[x]);
        if (KTYPE == 0) o[x] = ex2_approx(cexp * s);
        else if (KTYPE == 1) o[x] = fmaxf(s, 0.f);
        else o[x] = sqrt_approx(fmaxf(s, 0.f));
      }
      if (storer) bulk_wait_read0();                      // last tile's TMA stores have read the staging
      named_bar(1, kEpiWarps * 32);                       // staging free
#pragma unroll
      for (int x = 0; x < 32; x += 4)
        st_shared_v4(stage + stage_off(r, 32 * cq + x), o[x], o[x + 1], o[x + 2], o[x + 3]);
      fence_async_smem();                                 // generic-proxy writes -> visible to the TMA
      named_bar(1, kEpiWarps * 32);                       // tile staged
      if (use_tma_store && I * kTile >= rb) {
        // TMA clips the box past the last row / column (ragged edges); a tile starting above
        // the row range (negative box origin) takes the masked path below
        if (storer) {
#pragma unroll
          for (int c = 0; c < kTile / kBoxCols; ++c)
            tma_store_2d(&tmap_out, J * kTile + c * kBoxCols, I * kTile - rb, stage + c * kTile * 128, stream_out);
          bulk_commit();
        }
      } else {
        // n % 4 != 0 (row pitch not 16-byte aligned) or first partial tile row: masked stores
        const int jc = J * kTile + lane;
        for (int rr = warp; rr < kTile; rr += kEpiWarps) {
          const int gi = I * kTile + rr;
          if (gi < rb || gi >= re) continue;
          float* dst = out + (size_t)(gi - rb) * (size_t)n;
#pragma unroll
          for (int cc = 0; cc < kTile; cc += 32)
            if (jc + cc < n) __stcs(dst + jc + cc, ld_shared_f32(stage + stage_off(rr, lane + cc)));
        }
      }
    }
    if (storer) asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");   // all TMA stores complete
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
