// tbs_kernels.cuh — sm_100a kernels of the 2-body-statistics hot path.
//
// Paper: Pitaksirianan, Nouri & Tu, ICPP 2016 (/root/reference/PAPER.md, cited L<a>-<b>).
// The design keeps the paper's ideas that still hold on B200 and drops the rest
// (DESIGN.md §Kernels):
//   * SoA input (L338-341)                       -> loader writes [D][n_pad] fp32 SoA
//   * block tiling, Alg. 2 (L366-458)            -> triangular (anchor tile, partner chunk)
//                                                   work items over persistent CTAs
//   * anchor datum in registers, Alg. 3 (L465-511)-> KA anchors per thread (Cfg), packed in
//                                                   f32x2 register pairs (FADD2/FFMA2)
//   * partner block in cache (L499)              -> TMA bulk copy (cp.async.bulk) into
//                                                   shared memory, double-buffered on mbarriers,
//                                                   read as LDS.128 broadcasts
//   * privatised output, Fig. 3 (L722-782)       -> 32 lane-private u32 copies per CTA
//                                                   (conflict-free ATOMS), u64 flush
//   * Type-I register output (L704-709)          -> per-thread sign-bit counter
//   * Type-III global output (L709-712)          -> streaming float4 stores
//   * intra-block i<j (Alg. 2 l.9-12, Fig. 6)    -> predicated pairs on diagonal items
#pragma once
#include <cstdint>
#include "tbs_ptx.cuh"

namespace tbs {

#ifndef TBS_PUNROLL
#define TBS_PUNROLL 1                      // partner-quad loop unroll (software-pipelining freedom)
#endif
#ifndef TBS_SW_SQRT
#define TBS_SW_SQRT 0                      // float SDH: (partner q, anchor pair m) slots, bit 4q+m, whose
#endif                                     // square roots run on the FMA pipe (sqrt_sw2) instead of MUFU
constexpr int kThreads = 256;              // 8 warps per CTA
constexpr int kPUnroll = TBS_PUNROLL;
constexpr unsigned kSwSqrtMask = TBS_SW_SQRT;
#ifndef TBS_MQ_ORDER
#define TBS_MQ_ORDER 0                     // A/B only: 1 = anchor-major slots for every Op; 2, 3 = two-phase groups
#endif
constexpr int kMqOrder = TBS_MQ_ORDER;
#ifndef TBS_PARTNER_PATH
#define TBS_PARTNER_PATH 0                 // Fig. 9 ablation (A/B builds only): how partners reach the
#endif                                     // threads, see run_chunk
constexpr int kPartnerPath = TBS_PARTNER_PATH;
constexpr int kWarps = kThreads / 32;
constexpr int kPadAlign = 4096;            // SoA rows padded to a multiple of every anchor tile / chunk
constexpr uint32_t kMagic = 0x4B000000u;   // bits of 2^23: x + 2^23 (round-down) = 2^23 + floor(x)
constexpr float kMagicF = 8388608.0f;
constexpr int kNoAnchor = 0x7fffffff;      // masked anchor index (no partner is greater)

// Pair-engine configuration: KA anchors per thread (register-blocked, packed in KA/2
// f32x2 pairs), TP partners per staged chunk, MINB resident CTAs per SM that the
// register budget targets. Anchor tile TA = 256 * KA points.
template <int KA_, int TP_, int MINB_>
struct Cfg {
  static constexpr int KA = KA_, TP = TP_, MINB = MINB_, TA = kThreads * KA_, RATIO = TA / TP_;
  static_assert(KA_ % 2 == 0 && TP_ % 4 == 0 && TA % TP_ == 0 && kPadAlign % TA == 0, "bad pair-engine config");
};

// Work decomposition (host-computed). Anchor tiles I in [I0, I1) of TA points; for each,
// partner chunks J in [I*ratio, Mc) of TP points. Item count: sum_I (Mc - I*ratio).
struct Geom {
  int n;            // number of points
  int rb, re;       // anchor rows [rb, re)
  int I0, I1;       // anchor tiles
  int Mc;           // ceil(n / TP)
  int ratio;        // TA / TP
  int n_pad;        // SoA row stride (multiple of kPadAlign)
  long long items;  // total work items
  unsigned long long* trace;  // debug only (TBS_TRACE): per CTA {smid, t_start, t_end}, else nullptr
  unsigned long long* counter;  // work-queue head (zeroed by the loader's memset), in items
  long long chunk;              // items grabbed per atomic (0: static, one item per CTA)
};

__device__ __forceinline__ long long items_before(const Geom& g, long long I) {
  return (I - g.I0) * (long long)g.Mc - (long long)g.ratio * ((I * (I - 1) - (long long)g.I0 * (g.I0 - 1)) / 2);
}
__device__ __forceinline__ void item_to_tile(const Geom& g, long long it, int& I, int& J) {
  int lo = g.I0, hi = g.I1 - 1;
  while (lo < hi) {
    int mid = (lo + hi + 1) >> 1;
    if (items_before(g, mid) <= it) lo = mid; else hi = mid - 1;
  }
  I = lo;
  J = lo * g.ratio + (int)(it - items_before(g, lo));
}

// ------------------------------------------------------------------------------------
// a1: SoA loader. AoS [n][dim] -> SoA [D][n_pad] (pad coordinates and pad points = 0).
// Also zeroes `zero_words` u64 words at `zero` (the caller's output / partial copies),
// saving a separate memset launch, and reduces the bounding box of the points into
// `bbox` (zero-initialised): bbox[c] = max of ~ord(x_c), bbox[D + c] = max of ord(x_c),
// with ord() the order-preserving float -> u32 map; bbox[2D] |= 1 on a non-finite
// coordinate. The pair kernel uses it to prove that no distance can leave the
// histogram's guard rows, which lets it drop the clamp instruction.
// ------------------------------------------------------------------------------------
__device__ __forceinline__ uint32_t f2ord(float x) {
  const uint32_t b = __float_as_uint(x);
  return (b & 0x80000000u) ? ~b : (b | 0x80000000u);
}
__device__ __forceinline__ float ord2f(uint32_t o) {
  return __uint_as_float((o & 0x80000000u) ? (o & 0x7fffffffu) : ~o);
}

// `pad` is the coordinate value of pad points i >= n (0; +inf for kNN, so pad partners never
// enter a neighbour list). Coordinates c >= dim of real points (dim 1, 2 padded to D = 3) are 0
// and enter the bounding box as such. bbox[2D] bit 0: a non-finite coordinate; bit 1: a
// non-integer coordinate (TBS_VALIDATE under TBS_EXACT_LATTICE).
__global__ void soa_loader(const float* __restrict__ pts, int n, int dim, int n_pad, int D, float pad,
                           float* __restrict__ soa, unsigned long long* __restrict__ zero, long long zero_words,
                           uint32_t* __restrict__ bbox) {
  const long long stride = (long long)gridDim.x * blockDim.x;
  uint32_t lo[4] = {0u, 0u, 0u, 0u}, hi[4] = {0u, 0u, 0u, 0u}, bad = 0u;
  for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < n_pad; i += stride) {
    for (int c = 0; c < D; ++c) {
      float v = pad;
      if (i < n) {
        v = c < dim ? __ldg(pts + i * dim + c) : 0.0f;
        const uint32_t o = f2ord(v);
        lo[c] = max(lo[c], ~o);
        hi[c] = max(hi[c], o);
        bad |= (isfinite(v) ? 0u : 1u) | (v == rintf(v) ? 0u : 2u);
      }
      soa[(long long)c * n_pad + i] = v;
    }
  }
  for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < zero_words; i += stride) zero[i] = 0ull;
  if (bbox) {
    // warp shuffles, then the CTA's warps in shared memory, then ONE atomic per box word per
    // CTA (per-warp global atomics on the same 2D+1 words serialised in L2: ~0.1 ms at 1M)
    __shared__ uint32_t sb[9];
    if (threadIdx.x < 9) sb[threadIdx.x] = 0u;
    __syncthreads();
    for (int c = 0; c < D; ++c) {
      uint32_t a = lo[c], b = hi[c];
#pragma unroll
      for (int off = 16; off > 0; off >>= 1) {
        a = max(a, __shfl_xor_sync(0xffffffffu, a, off));
        b = max(b, __shfl_xor_sync(0xffffffffu, b, off));
      }
      if ((threadIdx.x & 31) == 0) {
        if (a) atomicMax(sb + c, a);
        if (b) atomicMax(sb + D + c, b);
      }
    }
#pragma unroll
    for (int off = 16; off > 0; off >>= 1) bad |= __shfl_xor_sync(0xffffffffu, bad, off);
    if ((threadIdx.x & 31) == 0 && bad) atomicOr(sb + 2 * D, bad);
    __syncthreads();
    if (threadIdx.x < 2 * D) {
      if (sb[threadIdx.x]) atomicMax(bbox + threadIdx.x, sb[threadIdx.x]);
    } else if (threadIdx.x == 2 * D && sb[2 * D]) {
      atomicOr(bbox + 2 * D, sb[2 * D]);
    }
  }
}

// The same for small problems (n_pad <= kSmallLoad): ONE 1024-thread CTA, D a template
// argument, 32-bit indices, reduction in shared memory, and the whole 64-byte box block
// written at the end, so the caller needs no memset before it (the small-problem path is
// latency-bound, BASELINE configs[0]; the general loader took 9.8 us there, ncu r02).
constexpr int kSmallLoad = 16384;
template <int D>
__global__ void __launch_bounds__(1024) soa_loader_small(const float* __restrict__ pts, int n, int dim, int n_pad, float pad,
                                                          float* __restrict__ soa, unsigned long long* __restrict__ zero,
                                                          int zero_words, uint32_t* __restrict__ bbox) {
  __shared__ uint32_t sb[16];
  if (threadIdx.x < 16) sb[threadIdx.x] = 0u;
  uint32_t lo[D], hi[D], bad = 0u;
#pragma unroll
  for (int c = 0; c < D; ++c) lo[c] = hi[c] = 0u;
#pragma unroll 4
  for (int i = threadIdx.x; i < n_pad; i += 1024) {
#pragma unroll
    for (int c = 0; c < D; ++c) {
      float v = pad;
      if (i < n) {
        v = c < dim ? __ldg(pts + i * dim + c) : 0.0f;
        const uint32_t o = f2ord(v);
        lo[c] = max(lo[c], ~o);
        hi[c] = max(hi[c], o);
        bad |= (isfinite(v) ? 0u : 1u) | (v == rintf(v) ? 0u : 2u);
      }
      soa[c * n_pad + i] = v;
    }
  }
  for (int i = threadIdx.x; i < zero_words; i += 1024) zero[i] = 0ull;
  __syncthreads();
#pragma unroll
  for (int c = 0; c < D; ++c) {
    uint32_t a = lo[c], b = hi[c];
#pragma unroll
    for (int off = 16; off > 0; off >>= 1) {
      a = max(a, __shfl_xor_sync(0xffffffffu, a, off));
      b = max(b, __shfl_xor_sync(0xffffffffu, b, off));
    }
    if ((threadIdx.x & 31) == 0) {
      if (a) atomicMax(sb + c, a);
      if (b) atomicMax(sb + D + c, b);
    }
  }
#pragma unroll
  for (int off = 16; off > 0; off >>= 1) bad |= __shfl_xor_sync(0xffffffffu, bad, off);
  if ((threadIdx.x & 31) == 0 && bad) atomicOr(sb + 2 * D, bad);
  __syncthreads();
  if (threadIdx.x < 16) bbox[threadIdx.x] = sb[threadIdx.x];
}

// Upper bound on any pair distance from the loader's bounding box (+inf if unknown): fp32 with
// a 1e-5 relative margin (the fp32 rounding of three squares, a sum and a square root is
// < 1e-6), far below the two guard bins the no-clamp test keeps.
__device__ __forceinline__ float bbox_diameter(const uint32_t* __restrict__ bbox, int D) {
  if (bbox == nullptr || (bbox[2 * D] & 1u) != 0u) return __int_as_float(0x7f800000);
  float s = 0.0f;
  for (int c = 0; c < D; ++c) {
    if (bbox[c] == 0u || bbox[D + c] == 0u) return __int_as_float(0x7f800000);
    const float e = __fsub_ru(ord2f(bbox[D + c]), ord2f(~bbox[c]));
    s = __fmaf_ru(e, e, s);
  }
  return __fmul_ru(__fsqrt_ru(s), 1.00001f);
}

// ------------------------------------------------------------------------------------
// Where the Type-I / Type-II flushes land (a9, a12). n == 0: the buffer p[0] (device-scope
// atomics): the caller's output, or under TBS_OUT_PEERS the call's local accumulator. n >= 1
// (push_peers, the second stage of the fused multi-GPU combine): every rank's buffer p[0..n)
// — local or mapped from a peer GPU over NVLink by CUDA IPC — gets the partial with a
// system-scope atomic add, so when all ranks' calls have completed each buffer holds the
// all-reduced sum without a separate collective.
// ------------------------------------------------------------------------------------
constexpr int kMaxPeers = 16;
struct OutSink {
  unsigned long long* p[kMaxPeers];
  int n;
  __device__ __forceinline__ void add(long long k, unsigned long long v) const {
    if (n == 0) {
      atomicAdd(p[0] + k, v);
    } else {
      for (int w = 0; w < n; ++w) red_sys_add_u64(p[w] + k, v);
    }
  }
  // After a CTA's last flush: order its remote adds before kernel completion is observed.
  __device__ __forceinline__ void fence() const {
    if (n != 0) __threadfence_system();
  }
};

// Fused multi-GPU combine folded into the pair kernel's tail (TBS_OUT_PEERS, single-launch
// output stages): every CTA's flush lands in the rank's local accumulator `acc` (device-scope
// atomics); each CTA then takes a ticket, and the LAST CTA of the grid adds the `words` of
// `acc` into every rank's buffer (`peers`, n >= 1: local or mapped from a peer GPU over
// NVLink) with system-scope atomics — the compute and its all-reduce exchange in ONE kernel.
// words == 0: no tail (the caller pushes with push_peers, or there are no peers).
struct TailPush {
  OutSink peers;
  const unsigned long long* acc;
  unsigned int* ticket;   // zeroed before the launch (a spare word of the bounding-box block)
  int words;
};

__device__ __forceinline__ void push_tail(const TailPush& t) {
  __shared__ unsigned int s_last;
  __threadfence();        // this CTA's flush atomics are visible device-wide before its ticket
  __syncthreads();
  if (threadIdx.x == 0) s_last = atomicAdd(t.ticket, 1u) == gridDim.x - 1 ? 1u : 0u;
  __syncthreads();
  if (s_last) {
    __threadfence();      // every other CTA's flush precedes its ticket: read acc from L2
    for (int k = threadIdx.x; k < t.words; k += blockDim.x) {
      const unsigned long long v = __ldcg(t.acc + k);
      if (v) t.peers.add(k, v);
    }
    t.peers.fence();
  }
}

// ------------------------------------------------------------------------------------
// Output-stage policies. Each provides:
//   smem_bytes()                    dynamic shared memory it needs (host and device)
//   init(smem), finish(smem)        zero / flush its private copies
//   after_item(smem, since)         flush early if a u32 counter could overflow
//   bias()                          value the squared-distance chain starts from
//   pair2<MASKED>(s2, pv, a0, a1)   consume two pairs (anchors a0, a1 vs partner pv);
//                                   under MASKED a pair counts only if pv > a
// ------------------------------------------------------------------------------------

// Type-II, float mode: bucket = min(floor(sqrt(s) / w), nb - 1) with R replicas per bin
// in shared memory, layout word[k * R + (lane & (R-1))]. R = 32: every lane owns a copy
// and the 32 lanes of an ATOMS hit 32 distinct banks (no conflicts, no same-address).
//
// Per pair: MUFU.SQRT, then for two pairs one FFMA2.RM  y = RD(q * (1/w) + 2^23) = 2^23 + k
// (the 1/w scale and the floor in one rounding; bits(y) = bits(2^23) + k), then per pair
// one ALU LEA.HI: (bits(y) << log2(4R)) | 4 lane_r, plus the CTA-uniform
// (smem base - (bits(2^23) << log2(4R))) fused as a uniform-register operand — no IMAD on
// the FMA pipe — and the ATOMS (red.shared.add.u32).
// The clamp k <= nb-1 (one FMNMX per pair) is dropped when the loader's bounding box
// proves k < nb + kGuard for every pair; guard rows are folded into nb-1 at the flush.
// LATTICE: exact integer bucketing max{k : (k m)^2 <= 4^j s} for integer-valued input.
constexpr int kGuard = 32;

extern __shared__ __align__(128) unsigned char tbs_smem[];  // dynamic smem; histogram at offset 0

// Histogram increment. TBS_BOUNDS_CHECK (debug builds: compute-sanitizer is not available on the
// GPU pool) traps if the address computed by the bucket / LEA.HI arithmetic leaves the histogram
// words of the dynamic shared memory (replicas, guard rows, trash row).
__device__ __forceinline__ void hist_inc(uint32_t a, long long hist_bytes) {
#ifdef TBS_BOUNDS_CHECK
  const uint32_t base = smem_addr(tbs_smem);
  if (a < base || (long long)(a - base) + 4 > hist_bytes || (a & 3u) != 0u) {
    printf("tbs bounds: smem increment at offset %lld outside [0, %lld) (block %d thread %d)\n",
           (long long)a - (long long)base, hist_bytes, (int)blockIdx.x, (int)threadIdx.x);
    __trap();
  }
#endif
  (void)hist_bytes;
  red_smem_inc(a);
}

// RANGED: bucket-range pass for nb beyond one shared-memory copy: only buckets
// [klo, klo + rows) are counted in this launch (one predicated ATOMS); the host runs
// ceil(nb / rows) passes over the triangle instead of falling back to global atomics.
template <int LOG2R, bool LATTICE, bool RANGED = false>
struct SdhSmemOp {
  static constexpr int R = 1 << LOG2R;
  int klo = 0;        // first bucket of this pass (RANGED)
  int nb;             // buckets
  int rows;           // rows allocated (nb, + kGuard in float mode)
  float inv_w;        // fp32(1 / w)                       (float mode)
  float scale;        // fp32(2^j / m)                     (lattice mode)
  float scale_up;     // fp32(2^j / m) * (1 + 2^-17), rounded up (lattice fast variant)
  float scale_b;      // fp32(2^j / m) * (1 + 2^-19), rounded up (lattice bias-only variant)
  int m, sh;          // w = m * 2^-j, sh = 2 j            (lattice mode)
  const OutSink* out; // global u64 output [nb] (or every rank's): the kernel's sink parameter
  float ymax;         // float: 2^23 + nb - 1 (clamp variant)
  int flush_every;    // items between overflow flushes

  // rows + 1: the last row is the trash row masked pairs increment (never flushed)
  __host__ __device__ long long smem_bytes() const { return (long long)(rows + 1) * R * 4; }

  __device__ __forceinline__ void init(unsigned char* smem) {
    uint32_t* h = reinterpret_cast<uint32_t*>(smem);
    for (int i = threadIdx.x; i < rows * R; i += kThreads) h[i] = 0u;
    ymax = kMagicF + (float)(nb - 1);
  }
  __device__ __forceinline__ float2 bias() const { return make_float2(0.f, 0.f); }
  // Kernel-uniform code variant, chosen once from the loader's bounding box:
  //   float mode:   0 = no clamp (every k < nb + kGuard is proven), 1 = clamp to nb-1;
  //   lattice mode: 4 = bias only, no fix-up and no clamp (see below; every bucket edge
  //                 the data can reach is far enough from the estimate's error),
  //                 0 = fp32 one-sided fix-up, no clamp (all products < 2^24 and every
  //                 estimate < nb + kGuard proven; not in bucket-range passes),
  //                 exact two-sided fix-up in 1 = fp32, 2 = 32-bit integers,
  //                 3 = 64-bit integers (general).
  static constexpr int kVariants = LATTICE ? 5 : 2;
  float mj;           // lattice: m * 2^-j (exact)
  __device__ __forceinline__ int variant(const uint32_t* bbox, int D) const {
    const float dmax = bbox_diameter(bbox, D);
    if (LATTICE) {
      const double smax = (double)dmax * (double)dmax;             // >= every s (integer data)
      const double S = smax * (double)(1ull << sh);                // 4^j s_max
      const double kmax = floor(sqrt(S) / (double)m) + 2.0;         // estimate + fix-up reach
      const double e = fmax(kmax, (double)(nb + 1)) * (double)m;
      // Bias-only variant: x = sqrt(4^j s) / m, k = floor(x). The estimate q c with
      // q = sqrt.approx(s) (|rel err| <= 2^-22, measured exhaustively over every integer
      // s < 2^24: tools/sqrt_bound.cu) and c = 2^j/m (1 + 2^-19) rounded up lies in
      // [x, x (1 + g)], g < 2^-18. Below the next edge, S = 4^j s <= X^2 - 1 with X = (k+1) m
      // (integers), so x <= (k+1)(1 - 1/(2 X^2)): floor(q c) = k whenever 2 X^2 g < 1,
      // i.e. X^2 < 2^17 for the largest X the bounding box allows.
      const double xmax = sqrt(S) / (double)m;
      const double X = (floor(xmax) + 1.0) * (double)m;
      if (!RANGED && smax < 16777216.0 && X * X < 131072.0 && xmax * (1.0 + 1.0 / 262144.0) + 2.0 < (double)(nb + kGuard))
        return 4;
      // One-sided fp32 variant 0 (pair2, V == 0). It needs: s exact in fp32 (smax < 2^23);
      // k0 = floor(q c_up) in {k, k + 1}, i.e. x (1 + 2^-16) < k + 2 for every reachable
      // x = sqrt(4^j s) / m (x < 2^15 leaves a 2x margin); e0 = k0 m 2^-j exact (k0 m < 2^24);
      // the sign of t = s - e0^2 exact — one FFMA: the product is exact inside it and a rounding
      // never flips a sign, s and e0^2 being multiples of 4^-j far above the underflow range —
      // and every estimate a valid row (no clamp). It does NOT need 4^j s < 2^24 (r02: the C4
      // lattice, w = 2^-6, X up to 14080, took the 32-bit integer variant for that reason).
      if (!RANGED && smax < 8388608.0 && xmax < 32768.0 && (kmax + 1.0) * (double)m < 16777216.0 &&
          xmax * (1.0 + 1.0 / 32768.0) + 2.0 < (double)(nb + kGuard))
        return 0;
      if (smax < 8388608.0 && S < 16777216.0 && e * e < 16777216.0) return 1;
      const double em = (double)(nb + 1) * (double)m;
      if (smax < 8388608.0 && S < 4294967296.0 && em * em < 4294967296.0) return 2;
      return 3;
    }
    return (dmax * inv_w < (float)(nb + kGuard - 2)) ? 0 : 1;
  }

  // Lattice bucket: s is an exact integer (< 2^24; < 2^23 on the 32-bit path). fp32
  // estimate k0 = floor(sqrt(s) 2^j / m), then one exact integer step each way against
  // (k m)^2 <= 4^j s. Returns the clamped bucket index.
  template <int V>
  __device__ __forceinline__ uint32_t lattice_bucket(float s) const {
    const float q = sqrt_approx(s);
    int k = min((int)(__float_as_uint(__fmaf_rd(q, scale, kMagicF)) - kMagic), nb);
    if (V == 3) {
      const unsigned long long S = (unsigned long long)__float2uint_rz(s) << sh;
      const unsigned long long e1 = (unsigned long long)(k + 1) * (unsigned long long)m;
      k += (e1 * e1 <= S) ? 1 : 0;
      const unsigned long long e0 = (unsigned long long)k * (unsigned long long)m;
      k -= (e0 * e0 > S) ? 1 : 0;
    } else {
      const uint32_t S = (__float_as_uint(__fadd_rn(s, kMagicF)) - kMagic) << sh;   // exact for s < 2^23
      const uint32_t e1 = (uint32_t)(k + 1) * (uint32_t)m;
      k += (e1 * e1 <= S) ? 1 : 0;
      const uint32_t e0 = (uint32_t)k * (uint32_t)m;
      k -= (e0 * e0 > S) ? 1 : 0;
    }
    return (uint32_t)min(k, nb - 1);
  }

  // Lattice, fp32 fix-up for two pairs: with e = k m 2^-j, e^2 - s = ((k m)^2 - 4^j s) / 4^j
  // is an integer < 2^24 scaled by a power of two, so one FFMA computes it exactly.
  __device__ __forceinline__ void lattice_bucket2_f32(float2 s, uint32_t& k0, uint32_t& k1) const {
    const float2 q = make_float2(sqrt_approx(s.x), sqrt_approx(s.y));
    const float2 y = __ffma2_rd(q, make_float2(scale, scale), make_float2(kMagicF, kMagicF));
    const float2 kf = __fadd2_rn(y, make_float2(-kMagicF, -kMagicF));
    const float2 e0 = __fmul2_rn(kf, make_float2(mj, mj));
    const float2 e1 = __fadd2_rn(e0, make_float2(mj, mj));
    const float2 ns = make_float2(-s.x, -s.y);
    const float2 d1 = __ffma2_rn(e1, e1, ns);
    const float2 d0 = __ffma2_rn(e0, e0, ns);
    const int b0 = (int)(__float_as_uint(y.x) - kMagic), b1 = (int)(__float_as_uint(y.y) - kMagic);
    k0 = (uint32_t)min(b0 + (d1.x <= 0.f ? 1 : 0) - (d0.x > 0.f ? 1 : 0), nb - 1);
    k1 = (uint32_t)min(b1 + (d1.y <= 0.f ? 1 : 0) - (d0.y > 0.f ? 1 : 0), nb - 1);
  }

  // Float mode (or the lattice bias-only variant, estimate scale c instead of 1/w): smem word
  // addresses of the buckets of two pairs from their square roots q.
  template <int V>
  __device__ __forceinline__ void float_addr2(float2 q, uint32_t& ad0, uint32_t& ad1, bool& in0, bool& in1) const {
    const float c = LATTICE ? scale_b : inv_w;
    float2 y = __ffma2_rd(q, make_float2(c, c), make_float2(kMagicF, kMagicF));
    if (!LATTICE && V == 1) {
      y.x = fminf(y.x, ymax);
      y.y = fminf(y.y, ymax);
    }
    // bits(y) = bits(2^23) + k. Funnel shift (bits << S) | (lo >> (32-S)) with S = log2(4R)
    // and lo = 4 lane_r << (32-S) gives 4 (k R + lane_r) + (bits(2^23) << S); the
    // CTA-uniform correction (smem base - (bits(2^23) << S)) is recomputed from the smem
    // symbol so ptxas fuses shift + add into one ALU LEA.HI with a uniform operand.
    constexpr int S = LOG2R + 2;
    const uint32_t lo = (uint32_t)((threadIdx.x & (R - 1)) * 4) << (32 - S);
    const uint32_t ub = smem_addr(tbs_smem) - ((kMagic + (RANGED ? (uint32_t)klo : 0u)) << S);
    ad0 = __funnelshift_l(lo, __float_as_uint(y.x), S) + ub;
    ad1 = __funnelshift_l(lo, __float_as_uint(y.y), S) + ub;
    if (RANGED) {
      in0 = __float_as_uint(y.x) - (kMagic + (uint32_t)klo) < (uint32_t)rows;
      in1 = __float_as_uint(y.y) - (kMagic + (uint32_t)klo) < (uint32_t)rows;
    }
  }

  // Float mode, unmasked pairs, square roots on the FMA pipe (the TBS_SW_SQRT slots).
  static constexpr bool kSwCapable = !LATTICE && !RANGED;
  // slot order of a partner group (run_chunk): anchor-major measured +1.0 % for float SDH at
  // 1M, but -7.4 % for the lattice variants at 4M and -20 % for bucket-range passes (65536
  // buckets at 1M: 491 vs 409 ms; profiles/r02_slot_order_ab.txt, r02_ablations.jsonl)
  static constexpr bool kAnchorMajor = !LATTICE && !RANGED;
  template <int V>
  __device__ __forceinline__ void pair2_sw(float2 s) {
    uint32_t ad0, ad1;
    bool in0 = true, in1 = true;
    float_addr2<V>(sqrt_sw2(s), ad0, ad1, in0, in1);
    hist_inc(ad0, smem_bytes());
    hist_inc(ad1, smem_bytes());
  }

  template <bool MASKED, int V>
  __device__ __forceinline__ void pair2(float2 s, int pv, int a0, int a1) {
    uint32_t ad0, ad1;
    bool in0 = true, in1 = true;
    if (!LATTICE || V == 4) {
      float_addr2<V>(make_float2(sqrt_approx(s.x), sqrt_approx(s.y)), ad0, ad1, in0, in1);
    } else if (V == 0) {
      // Lattice, fast variant. The estimate uses a scale rounded UP by 2^-17, far above the
      // sqrt.approx + rounding error (~2^-22) and far below 1/x (x = sqrt(4^j s)/m < 2^15),
      // so k0 = floor(estimate) is k or k + 1, never less. One exact check decides:
      //   e0 = k0 m 2^-j  (one FFMA: (2^23 + k0) mj - 2^23 mj, exact as k0 m < 2^24)
      //   t  = s - e0^2   (one FFMA; its sign is exact: -0 never arises, t = 0 is a tie -> k0)
      // and t < 0 (k0 = k + 1) subtracts one from bits(y) (the sign word >> 31, arithmetic,
      // is -1) before the same LEA.HI addressing as float mode.
      const float2 q = make_float2(sqrt_approx(s.x), sqrt_approx(s.y));
      const float2 y = __ffma2_rd(q, make_float2(scale_up, scale_up), make_float2(kMagicF, kMagicF));
      const float nmj = -kMagicF * mj;
      const float2 e0 = __ffma2_rn(y, make_float2(mj, mj), make_float2(nmj, nmj));
      const float2 t = __ffma2_rn(make_float2(-e0.x, -e0.y), e0, s);
      constexpr int S = LOG2R + 2;
      const uint32_t lo = (uint32_t)((threadIdx.x & (R - 1)) * 4) << (32 - S);
      const uint32_t ub = smem_addr(tbs_smem) - (kMagic << S);
      const uint32_t b0 = __float_as_uint(y.x) + (uint32_t)(__float_as_int(t.x) >> 31);   // bits(2^23) + k
      const uint32_t b1 = __float_as_uint(y.y) + (uint32_t)(__float_as_int(t.y) >> 31);
      ad0 = __funnelshift_l(lo, b0, S) + ub;
      ad1 = __funnelshift_l(lo, b1, S) + ub;
    } else {
      uint32_t k0, k1;
      if (V == 1) {
        lattice_bucket2_f32(s, k0, k1);
      } else {
        k0 = lattice_bucket<V>(s.x);
        k1 = lattice_bucket<V>(s.y);
      }
      if (RANGED) {
        k0 -= (uint32_t)klo;
        k1 -= (uint32_t)klo;
        in0 = k0 < (uint32_t)rows;
        in1 = k1 < (uint32_t)rows;
      }
      const uint32_t lb = smem_addr(tbs_smem) + (uint32_t)((threadIdx.x & (R - 1)) * 4);
      ad0 = (k0 << (LOG2R + 2)) + lb;
      ad1 = (k1 << (LOG2R + 2)) + lb;
    }
    if (RANGED || MASKED) {
      // Masked pairs (i >= j, pad partners: their distance can leave the histogram) and
      // out-of-pass buckets increment the lane's word of the trash row `rows` instead: no
      // branch (a predicated ATOMS becomes BSSY/BRA/BSYNC), the same ATOMS.POPC.INC, and the
      // address stays inside the allocation.
      const uint32_t trash = smem_addr(tbs_smem) + (uint32_t)(((rows << LOG2R) + (threadIdx.x & (R - 1))) * 4);
      const bool c0 = in0 && (!MASKED || pv > a0), c1 = in1 && (!MASKED || pv > a1);
      hist_inc(c0 ? ad0 : trash, smem_bytes());
      hist_inc(c1 ? ad1 : trash, smem_bytes());
    } else {
      hist_inc(ad0, smem_bytes());
      hist_inc(ad1, smem_bytes());
    }
  }

  // Sum the R replicas of each bin and add to the global u64 output: one thread per bin reads
  // its R words in a rotated order r = (j + (t >> (5 - LOG2R))) mod R, so at every step j the
  // 32 lanes of a warp hit 32 distinct banks (bins t and t + 32/R differ in r), and zeroes them.
  // Independent loads instead of a dependent shuffle chain per bin: the flush was ~40 % of a
  // small (N = 4096) launch with the segmented-shuffle form (ncu source view, r02).
  // (Used for the final flush only: inside the item loop, the divergent per-thread loop cost the
  // hot loop its uniform-datapath addressing and 7 % at N = 1M on B200 — the mid-kernel
  // overflow flush keeps the warp-synchronous form below.)
  __device__ void flush(unsigned char* smem) {
    uint32_t* h = reinterpret_cast<uint32_t*>(smem);
    const int t = threadIdx.x & 31;
    const int rot = t >> (5 - LOG2R);
    for (int k = threadIdx.x; k < rows; k += kThreads) {
      unsigned long long v = 0;
#pragma unroll 8
      for (int j = 0; j < R; ++j) {
        const int w = k * R + ((j + rot) & (R - 1));
        v += h[w];
        h[w] = 0u;
      }
      if (v != 0ull) {
        const int kk = k + (RANGED ? klo : 0);
#ifdef TBS_BOUNDS_CHECK
        if (kk < 0) { printf("tbs bounds: flush bucket %d < 0\n", kk); __trap(); }
#endif
        out->add(kk < nb ? kk : nb - 1, v);
      }
    }
  }
  // Mid-kernel overflow flush: segmented shuffle-sum of each bin's R replicas (warp-uniform
  // loop, so the item loop around it keeps its uniform registers).
  __device__ void flush_in_loop(unsigned char* smem) {
    uint32_t* h = reinterpret_cast<uint32_t*>(smem);
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const int total = rows * R;
    for (int e0 = warp * 32; e0 < total; e0 += kWarps * 32) {
      const int e = e0 + lane;
      unsigned long long v = 0;
      if (e < total) { v = h[e]; h[e] = 0u; }
#pragma unroll
      for (int off = 1; off < R; off <<= 1) v += __shfl_xor_sync(0xffffffffu, v, off);
      if ((lane & (R - 1)) == 0 && v != 0ull && e < total) {
        const int k = (e >> LOG2R) + (RANGED ? klo : 0);
        out->add(k < nb ? k : nb - 1, v);
      }
    }
  }
  __device__ __forceinline__ void after_group() {}
  __device__ __forceinline__ void after_item(unsigned char* smem, int& since) {
    if (++since >= flush_every) {
      flush_in_loop(smem);
      __syncthreads();
      since = 0;
    }
  }
  __device__ __forceinline__ void finish(unsigned char* smem) {
    flush(smem);
    out->fence();
  }
};

// Type-II, partially privatised GLOBAL histogram (large nb, or forced): G u64 copies in
// global memory (L2-resident), CTA b adds into copy b % G; a reduce kernel sums them.
template <bool LATTICE>
struct SdhGlobalOp {
  int nb;
  float inv_w, scale;
  int m, sh;
  int G;
  unsigned long long* part;  // [G][nb]
  unsigned long long* mine;
  int flush_every;           // unused
  const OutSink* out;        // unused (the reduce kernel writes the sink)

  static constexpr bool kSwCapable = false;
  static constexpr bool kAnchorMajor = false;   // slot order (run_chunk; r02 A/B)
  __host__ __device__ long long smem_bytes() const { return 0; }
  __device__ __forceinline__ void init(unsigned char*) { mine = part + (size_t)(blockIdx.x % G) * nb; }
  __device__ __forceinline__ float2 bias() const { return make_float2(0.f, 0.f); }
  __device__ __forceinline__ int bucket(float s) const {
    int k;
    if (!LATTICE) {
      k = (int)(__float_as_uint(__fmaf_rd(sqrt_approx(s), inv_w, kMagicF)) - kMagic);
    } else {
      uint32_t si = __float2uint_rz(s);
      k = min((int)(__float_as_uint(__fmaf_rd(sqrt_approx(s), scale, kMagicF)) - kMagic), nb);
      unsigned long long S = (unsigned long long)si << sh;
      unsigned long long e1 = (unsigned long long)(k + 1) * (unsigned long long)m;
      k += (e1 * e1 <= S) ? 1 : 0;
      unsigned long long e0 = (unsigned long long)k * (unsigned long long)m;
      k -= (e0 * e0 > S) ? 1 : 0;
    }
    return min(k, nb - 1);
  }
  static constexpr int kVariants = 1;
  __device__ __forceinline__ int variant(const uint32_t*, int) const { return 0; }
  template <bool MASKED, int V>
  __device__ __forceinline__ void pair2(float2 s, int pv, int a0, int a1) {
    unsigned long long* p0 = mine + bucket(s.x);
    unsigned long long* p1 = mine + bucket(s.y);
    if (MASKED) {
      red_gmem_inc64_gt(p0, pv, a0);
      red_gmem_inc64_gt(p1, pv, a1);
    } else {
      red_gmem_inc64(p0);
      red_gmem_inc64(p1);
    }
  }
  __device__ __forceinline__ void after_group() {}
  __device__ __forceinline__ void after_item(unsigned char*, int&) {}
  __device__ __forceinline__ void finish(unsigned char*) {}
};

// Type-I 2PCF count: t = s - r^2 is formed inside the FMA chain (bias = -r^2), and the
// count adds the sign bit of t: [s < r^2] with no compare instruction.
struct PcfOp {
  float r2;
  const OutSink* out;        // u64 count (or every rank's): the kernel's sink parameter
  uint32_t c;                // per-item counter (<= KA * TP)
  unsigned long long total;  // per-thread running total
  static constexpr bool kSwCapable = false;
  static constexpr bool kAnchorMajor = false;   // slot order (run_chunk; r02 A/B)

  __host__ __device__ long long smem_bytes() const { return 0; }
  __device__ __forceinline__ void init(unsigned char*) { c = 0u; total = 0ull; }
  __device__ __forceinline__ float2 bias() const { return make_float2(-r2, -r2); }
  static constexpr int kVariants = 1;
  __device__ __forceinline__ int variant(const uint32_t*, int) const { return 0; }
  template <bool MASKED, int V>
  __device__ __forceinline__ void pair2(float2 t, int pv, int a0, int a1) {
    uint32_t s0 = __float_as_uint(t.x) >> 31, s1 = __float_as_uint(t.y) >> 31;
    if (MASKED) {
      s0 = (pv > a0) ? s0 : 0u;
      s1 = (pv > a1) ? s1 : 0u;
    }
    c += s0 + s1;
  }
  __device__ __forceinline__ void after_group() {}
  __device__ __forceinline__ void after_item(unsigned char*, int&) {
    total += c;
    c = 0u;
  }
  __device__ void finish(unsigned char* smem) {
    total += c;
    unsigned long long v = total;
#pragma unroll
    for (int off = 16; off > 0; off >>= 1) v += __shfl_xor_sync(0xffffffffu, v, off);
    unsigned long long* red = reinterpret_cast<unsigned long long*>(smem);  // >= kWarps * 8 bytes (partner buffers)
    __syncthreads();
    if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = v;
    __syncthreads();
    if (threadIdx.x == 0) {
      unsigned long long s = 0;
      for (int w = 0; w < kWarps; ++w) s += red[w];
      if (s) out->add(0, s);
      out->fence();
    }
  }
};

// Type-I kernel-density pair sum (NEXT-2): S = sum_{i<j} exp(-gamma s). Per pair one FMUL
// (x = -gamma log2(e) s, packed) and one MUFU.EX2; per-thread fp32 partial over one
// partner group (4 partners x KA anchors), folded into a Kahan-compensated fp32 running sum
// (error ~ 2u of the total), doubles from the CTA reduction on.
struct KdeOp {
  float c;                  // -gamma * log2(e)
  double* sum;              // global output (zeroed by the loader)
  float2 part;              // current group partial (two lanes of the packed pair)
  float tot, comp;          // Kahan running sum
  const OutSink* out;       // unused
  static constexpr bool kSwCapable = false;
  static constexpr bool kAnchorMajor = true;   // slot order (run_chunk; r02 A/B)
  __host__ __device__ long long smem_bytes() const { return 0; }
  __device__ __forceinline__ void init(unsigned char*) {
    part = make_float2(0.f, 0.f);
    tot = 0.f;
    comp = 0.f;
  }
  __device__ __forceinline__ float2 bias() const { return make_float2(0.f, 0.f); }
  static constexpr int kVariants = 1;
  __device__ __forceinline__ int variant(const uint32_t*, int) const { return 0; }
  template <bool MASKED, int V>
  __device__ __forceinline__ void pair2(float2 s, int pv, int a0, int a1) {
    const float2 x = __fmul2_rn(s, make_float2(c, c));
    float2 e = make_float2(ex2_approx(x.x), ex2_approx(x.y));
    if (MASKED) {
      e.x = (pv > a0) ? e.x : 0.f;
      e.y = (pv > a1) ? e.y : 0.f;
    }
    part = __fadd2_rn(part, e);
  }
  __device__ __forceinline__ void after_group() {
    const float y = (part.x + part.y) - comp;
    const float t = tot + y;
    comp = (t - tot) - y;
    tot = t;
    part = make_float2(0.f, 0.f);
  }
  __device__ __forceinline__ void after_item(unsigned char*, int&) {}
  __device__ void finish(unsigned char* smem) {
    double v = (double)tot - (double)comp;
#pragma unroll
    for (int off = 16; off > 0; off >>= 1) v += __shfl_xor_sync(0xffffffffu, v, off);
    double* red = reinterpret_cast<double*>(smem);
    __syncthreads();
    if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = v;
    __syncthreads();
    if (threadIdx.x == 0) {
      double t = 0.0;
      for (int w = 0; w < kWarps; ++w) t += red[w];
      atomicAdd(sum, t);
    }
  }
};

// ------------------------------------------------------------------------------------
// a2-a10: the pair engine. Persistent CTAs walk a contiguous range of the linearised
// triangular item list. Per item: anchors (KA per thread) in registers, partner chunk
// staged by TMA into a double-buffered smem slot, every (anchor, partner) pair evaluated
// as packed f32x2 arithmetic, the Op consumes the squared distances.
// ------------------------------------------------------------------------------------
template <int D, int TP>
__device__ __forceinline__ void issue_chunk(const float* __restrict__ soa, const Geom& g, int J, float* dst,
                                            uint32_t bar) {
  mbar_arrive_expect_tx(bar, D * TP * 4);
#pragma unroll
  for (int c = 0; c < D; ++c)
    bulk_g2s(smem_addr(dst + c * TP), soa + (long long)c * g.n_pad + (long long)J * TP, TP * 4, bar);
}

template <class Op, int D, class C, bool MASKED, int V>
__device__ __forceinline__ void run_chunk(Op& op, const float* __restrict__ B, const float2 (&na)[D][C::KA / 2],
                                          const Geom& g, int I, int p0, int cnt) {
  // masked items only: anchor index or kNoAnchor outside [rb, re) (built here so the
  // registers are not live in the unmasked loop)
  int aidx[C::KA];
  if (MASKED) {
#pragma unroll
    for (int k = 0; k < C::KA; ++k) {
      const int a = I * C::TA + k * kThreads + (int)threadIdx.x;
      aidx[k] = (a >= g.rb && a < g.re) ? a : kNoAnchor;
    }
  }
  const int n = g.n;
  // Partner path (the paper's Fig. 9 comparison, L1183-1221; product = 0):
  //   0  chunk staged in shared memory by TMA bulk copy, read as LDS.128 broadcasts (B = smem);
  //   1  Alg. 4 register sharing: each lane loads one partner per 32 from global memory (L1)
  //      and the warp broadcasts it with 3 SHFL per partner (B = global chunk);
  //   2  read-only L1 path: LDG.128 broadcasts straight from the global SoA (B = global chunk).
  float sh[D];
#pragma unroll kPUnroll
  for (int p = 0; p < cnt; p += 4) {
    float c4[D][4];
    if constexpr (kPartnerPath == 0) {
#pragma unroll
      for (int c = 0; c < D; ++c) {
        const float4 v = *reinterpret_cast<const float4*>(B + c * C::TP + p);
        c4[c][0] = v.x; c4[c][1] = v.y; c4[c][2] = v.z; c4[c][3] = v.w;
      }
    } else if constexpr (kPartnerPath == 2) {
#pragma unroll
      for (int c = 0; c < D; ++c) {
        const float4 v = __ldg(reinterpret_cast<const float4*>(B + (long long)c * g.n_pad + p));
        c4[c][0] = v.x; c4[c][1] = v.y; c4[c][2] = v.z; c4[c][3] = v.w;
      }
    } else {
      if ((p & 31) == 0) {
#pragma unroll
        for (int c = 0; c < D; ++c) sh[c] = __ldg(B + (long long)c * g.n_pad + p + (threadIdx.x & 31));
      }
#pragma unroll
      for (int c = 0; c < D; ++c)
#pragma unroll
        for (int q = 0; q < 4; ++q) c4[c][q] = __shfl_sync(0xffffffffu, sh[c], (p & 31) + q);
    }
    if constexpr (kMqOrder >= 2 && !(Op::kSwCapable && kSwSqrtMask != 0u)) {
      // A/B: two phases over PH slots (anchor-major): all squared distances, then all outputs
      constexpr int NS = 4 * (C::KA / 2), PH = kMqOrder == 2 ? NS : 4;
#pragma unroll
      for (int base = 0; base < NS; base += PH) {
        float2 sv[PH];
#pragma unroll
        for (int j = 0; j < PH; ++j) {
          const int q = (base + j) % 4, m = (base + j) / 4;
          float2 d = __fadd2_rn(na[0][m], make_float2(c4[0][q], c4[0][q]));
          sv[j] = __ffma2_rn(d, d, op.bias());
#pragma unroll
          for (int c = 1; c < D; ++c) {
            d = __fadd2_rn(na[c][m], make_float2(c4[c][q], c4[c][q]));
            sv[j] = __ffma2_rn(d, d, sv[j]);
          }
        }
#pragma unroll
        for (int j = 0; j < PH; ++j) {
          const int q = (base + j) % 4, m = (base + j) / 4;
          const int pv = MASKED ? ((p0 + p + q < n) ? p0 + p + q : -1) : 0;
          op.template pair2<MASKED, V>(sv[j], pv, MASKED ? aidx[2 * m] : 0, MASKED ? aidx[2 * m + 1] : 0);
        }
      }
      op.after_group();
      continue;
    }
#pragma unroll
    for (int qm = 0; qm < 4 * (C::KA / 2); ++qm) {
      // partner q, anchor pair m: partner-major or anchor-major — the order ptxas schedules the
      // 4 x KA/2 independent chains in (per Op, measured; TBS_MQ_ORDER=1 forces anchor-major)
      constexpr bool am = Op::kAnchorMajor || kMqOrder == 1;
      constexpr int M = C::KA / 2;
      int q = am ? qm % 4 : qm / M;
      int m = am ? qm / 4 : qm % M;
      if constexpr (kMqOrder == 4 && M % 2 == 0) {   // A/B: 2 x 2 blocks (anchor pairs x partners)
        const int blk = qm / 4, in = qm % 4;
        m = (blk / 2) * 2 + in / 2;
        q = (blk % 2) * 2 + in % 2;
      }
      if constexpr (kMqOrder == 5) {                  // A/B: diagonal
        m = qm % M;
        q = (qm / M + qm % M) % 4;
      }
      int pv = 0;
      if (MASKED) pv = (p0 + p + q < n) ? p0 + p + q : -1;
      {
        float2 d = __fadd2_rn(na[0][m], make_float2(c4[0][q], c4[0][q]));
        float2 s = __ffma2_rn(d, d, op.bias());
#pragma unroll
        for (int c = 1; c < D; ++c) {
          d = __fadd2_rn(na[c][m], make_float2(c4[c][q], c4[c][q]));
          s = __ffma2_rn(d, d, s);
        }
        if constexpr (Op::kSwCapable && !MASKED && kSwSqrtMask != 0u && V <= 1) {
          if ((kSwSqrtMask >> (q * 4 + m)) & 1u) {   // resolved at compile time (q, m unrolled)
            op.template pair2_sw<V>(s);
            continue;
          }
        }
        op.template pair2<MASKED, V>(s, pv, MASKED ? aidx[2 * m] : 0, MASKED ? aidx[2 * m + 1] : 0);
      }
    }
    op.after_group();
  }
}

// VSET: bit v set = code variant v is compiled into this instantiation. A launch whose
// kernel-uniform variant is not in VSET exits at once, so a variant with a smaller register
// footprint can be compiled (and made resident) on its own and launched beside the rest.
template <class Op, int D, class C, int VSET = 0x1F>
__global__ void __launch_bounds__(kThreads, C::MINB) pair_kernel(const float* __restrict__ soa, Geom g, Op op,
                                                            const uint32_t* __restrict__ bbox,
                                                            const __grid_constant__ OutSink sink,
                                                            const __grid_constant__ TailPush tail) {
  unsigned char* smem = tbs_smem;
  const long long hbytes = (op.smem_bytes() + 127) & ~127ll;
  float* bufs = reinterpret_cast<float*>(smem + hbytes);
  uint64_t* bars = reinterpret_cast<uint64_t*>(smem + hbytes + 2 * D * C::TP * 4);
  const uint32_t bar0 = smem_addr(bars), bar1 = smem_addr(bars + 1);
  const int tid = threadIdx.x;

  unsigned long long t_start = 0;
  if (g.trace != nullptr && tid == 0) asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t_start));
  op.out = &sink;   // (param space: the Op stays small, its copy lives in registers)
  op.init(smem);
  // kernel-uniform variant, computed by every thread from the same box (provably uniform: the
  // item loop's addressing stays on the uniform datapath)
  const int variant = op.variant(bbox, D);
  if (!((VSET >> variant) & 1)) return;   // CTA-uniform: another launch owns this variant
  if (tid == 0) {
    mbar_init(bar0, 1);
    mbar_init(bar1, 1);
    fence_mbar_init();
  }
  __syncthreads();

  // Dynamic work distribution: CTAs grab chunks of g.chunk consecutive items from a global
  // counter, so every CTA runs until the whole triangle is done (the warp arbiter favours
  // some CTAs of an SM over others; a static split left SMs with one straggler CTA).
  // Thread 0 decides the NEXT item one item ahead (to prefetch its partner chunk) and
  // publishes it through a parity-double-buffered shared slot.
  __shared__ long long s_it[2];
  __shared__ int s_I[2], s_J[2];
  long long it, chunk_end = 0;
  int I = 0, J = 0;
  // g.chunk == 0: one item per CTA (grid == items, small problems): item = blockIdx.x, no queue
  if (tid == 0) {
    it = g.chunk > 0 ? (long long)atomicAdd(g.counter, (unsigned long long)g.chunk) : (long long)blockIdx.x;
    if (it < g.items) {
      chunk_end = g.chunk > 0 ? min(it + g.chunk, g.items) : it + 1;
      item_to_tile(g, it, I, J);
      if (kPartnerPath == 0) issue_chunk<D, C::TP>(soa, g, J, bufs, bar0);
    }
    s_it[0] = it; s_I[0] = I; s_J[0] = J;
  }
  __syncthreads();
  it = s_it[0]; I = s_I[0]; J = s_J[0];
  if (it < g.items) {
    int curI = -1;
    uint32_t phase = 0u;  // bit s = parity of buffer s
    int since = 0;
    int s = 0;
    float2 na[D][C::KA / 2];  // negated anchor coordinates, packed (a_{2m}, a_{2m+1})
    while (true) {
      if (tid == 0) {
        long long nit = it + 1;
        int nI = I, nJ = J + 1;
        if (nit < chunk_end) {
          if (nJ == g.Mc) { nI = I + 1; nJ = nI * C::RATIO; }
        } else {
          nit = g.chunk > 0 ? (long long)atomicAdd(g.counter, (unsigned long long)g.chunk) : g.items;
          if (nit < g.items) {
            chunk_end = min(nit + g.chunk, g.items);
            item_to_tile(g, nit, nI, nJ);
          }
        }
        if (kPartnerPath == 0 && nit < g.items) issue_chunk<D, C::TP>(soa, g, nJ, bufs + (s ^ 1) * D * C::TP, s ? bar0 : bar1);
        s_it[s ^ 1] = nit; s_I[s ^ 1] = nI; s_J[s ^ 1] = nJ;
      }
      if (I != curI) {
        curI = I;
#pragma unroll
        for (int k = 0; k < C::KA; ++k) {
          const int a = I * C::TA + k * kThreads + tid;
#pragma unroll
          for (int c = 0; c < D; ++c) {
            const float v = -__ldg(soa + (long long)c * g.n_pad + a);
            if (k & 1) na[c][k >> 1].y = v; else na[c][k >> 1].x = v;
          }
        }
      }
      if (kPartnerPath == 0) {
        mbar_wait(s ? bar1 : bar0, (phase >> s) & 1u);
        phase ^= 1u << s;
      }
      const float* B = kPartnerPath == 0 ? bufs + s * D * C::TP : soa + (long long)J * C::TP;
      const int p0 = J * C::TP;
      const int cnt = min(C::TP, g.n - p0);
      const bool fast =
          (I * C::TA >= g.rb) && ((I + 1) * C::TA <= g.re) && (p0 >= (I + 1) * C::TA) && (cnt == C::TP);
      if constexpr (Op::kVariants > 4 && (VSET & 16)) {
        if (variant == 4) {
          if (fast) run_chunk<Op, D, C, false, 4>(op, B, na, g, I, p0, cnt);
          else run_chunk<Op, D, C, true, 4>(op, B, na, g, I, p0, cnt);
          goto item_done;
        }
      }
      if constexpr (Op::kVariants > 3 && (VSET & 8)) {
        if (variant == 3) {
          if (fast) run_chunk<Op, D, C, false, 3>(op, B, na, g, I, p0, cnt);
          else run_chunk<Op, D, C, true, 3>(op, B, na, g, I, p0, cnt);
          goto item_done;
        }
      }
      if constexpr (Op::kVariants > 2 && (VSET & 4)) {
        if (variant == 2) {
          if (fast) run_chunk<Op, D, C, false, 2>(op, B, na, g, I, p0, cnt);
          else run_chunk<Op, D, C, true, 2>(op, B, na, g, I, p0, cnt);
          goto item_done;
        }
      }
      if constexpr (Op::kVariants > 1 && (VSET & 2)) {
        if (variant == 1) {
          if (fast) run_chunk<Op, D, C, false, 1>(op, B, na, g, I, p0, cnt);
          else run_chunk<Op, D, C, true, 1>(op, B, na, g, I, p0, cnt);
          goto item_done;
        }
      }
      if constexpr (VSET & 1) {
        if (fast) run_chunk<Op, D, C, false, 0>(op, B, na, g, I, p0, cnt);
        else run_chunk<Op, D, C, true, 0>(op, B, na, g, I, p0, cnt);
      }
      goto item_done;  // (keeps the label referenced for single-variant ops)
    item_done:
      __syncthreads();
      op.after_item(smem, since);
      s ^= 1;
      it = s_it[s];
      I = s_I[s];
      J = s_J[s];
      if (it >= g.items) break;
    }
  }
  __syncthreads();
  op.finish(smem);
  if (g.trace != nullptr && tid == 0) {
    unsigned long long t_end;
    uint32_t smid;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t_end));
    asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
    g.trace[3 * blockIdx.x] = smid;
    g.trace[3 * blockIdx.x + 1] = t_start;
    g.trace[3 * blockIdx.x + 2] = t_end;
  }
  if (tail.words > 0) push_tail(tail);   // kernel-uniform (a launch parameter)
}

// Fused multi-GPU combine, second stage (TBS_OUT_PEERS): the call's kernels accumulated this
// rank's partial in a local buffer with device-scope atomics; one thread per word adds it into
// every rank's output buffer with system-scope atomics (words x ranks remote adds per rank,
// instead of one add per flushing CTA), then fences them before the kernel completes.
__global__ void push_peers(const unsigned long long* __restrict__ acc, int words, OutSink out) {
  for (int k = blockIdx.x * blockDim.x + threadIdx.x; k < words; k += gridDim.x * blockDim.x) {
    const unsigned long long v = acc[k];
    if (v) out.add(k, v);
  }
  out.fence();
}

// Small problems (BASELINE configs[0], N = 4096): one work item per CTA and the loader fused
// in. Each CTA reads its anchors and its partner chunk straight from the caller's AoS points
// (the chunk, D x TP floats, is one contiguous AoS span, transposed into the shared-memory
// SoA layout run_chunk reads), so the call is one memset of the output plus this launch
// instead of a loader launch plus the pair kernel (the loader was ~7 us of a ~20 us step).
// No bounding box exists here: float SDH takes the clamp variant V.
// WriteBack (host-buffer calls): the last CTA to finish copies the `words` u64 of the result
// at `src` to mapped page-locked host memory `dst` (ticket zeroed before the launch).
// Then it stores `seq` to the mapped host word `flag` (after a system fence), which the host
// polls instead of waiting in a stream synchronisation.
// rezero: the last CTA also zeroes `src` and the ticket after the write-back, so the caller's
// cached scratch is zero again for its next call (no memset or copy kernel before the launch).
struct WriteBack {
  unsigned long long* dst = nullptr;
  unsigned long long* src = nullptr;
  unsigned int* ticket = nullptr;
  int words = 0;
  unsigned int* flag = nullptr;
  unsigned int seq = 0;
  int rezero = 0;
};

template <class Op, int D, class C, int V>
__global__ void __launch_bounds__(kThreads, C::MINB) pair_kernel_small(const float* __restrict__ pts, int dim, Geom g,
                                                                  Op op, const __grid_constant__ OutSink sink,
                                                                  const WriteBack wb) {
  unsigned char* smem = tbs_smem;
  const long long hbytes = (op.smem_bytes() + 127) & ~127ll;
  float* B = reinterpret_cast<float*>(smem + hbytes);
  const int tid = threadIdx.x;
  op.out = &sink;
  op.init(smem);
  int I, J;
  item_to_tile(g, (long long)blockIdx.x, I, J);
  const int p0 = J * C::TP;
  // Programmatic dependent launch (host-buffer calls: this grid may start while the copy
  // kernel that brings the points is still running): everything above overlaps it; wait for
  // its completion before the first read of the points. A no-op without the launch attribute.
  asm volatile("griddepcontrol.wait;" ::: "memory");
  for (int p = tid; p < C::TP; p += kThreads) {
    const long long j = p0 + p;
#pragma unroll
    for (int c = 0; c < D; ++c) B[c * C::TP + p] = (j < g.n && c < dim) ? __ldg(pts + j * dim + c) : 0.0f;
  }
  float2 na[D][C::KA / 2];
#pragma unroll
  for (int k = 0; k < C::KA; ++k) {
    const long long a = (long long)I * C::TA + k * kThreads + tid;
#pragma unroll
    for (int c = 0; c < D; ++c) {
      const float v = (a < g.n && c < dim) ? -__ldg(pts + a * dim + c) : 0.0f;
      if (k & 1) na[c][k >> 1].y = v; else na[c][k >> 1].x = v;
    }
  }
  __syncthreads();
  const int cnt = min(C::TP, g.n - p0);
  const bool fast = (I * C::TA >= g.rb) && ((I + 1) * C::TA <= g.re) && (p0 >= (I + 1) * C::TA) && (cnt == C::TP);
  if (fast) run_chunk<Op, D, C, false, V>(op, B, na, g, I, p0, cnt);
  else run_chunk<Op, D, C, true, V>(op, B, na, g, I, p0, cnt);
  __syncthreads();
  op.finish(smem);
  if (wb.dst != nullptr) {
    __shared__ unsigned int s_last;
    __threadfence();                       // this CTA's output atomics before its ticket
    __syncthreads();
    if (tid == 0) s_last = atomicAdd(wb.ticket, 1u) == gridDim.x - 1 ? 1u : 0u;
    __syncthreads();
    if (s_last) {
      __threadfence();
      for (int k = tid; k < wb.words; k += kThreads) {
        wb.dst[k] = __ldcg(wb.src + k);
        if (wb.rezero) wb.src[k] = 0ull;
      }
      __threadfence_system();
      __syncthreads();
      if (tid == 0 && wb.rezero) *wb.ticket = 0u;   // every other CTA took its ticket before this one
      if (tid == 0 && wb.flag != nullptr) {
        *reinterpret_cast<volatile unsigned int*>(wb.flag) = wb.seq;
        __threadfence_system();
      }
    }
  }
}

// Host-buffer small calls: copy the points from mapped page-locked host memory and zero the
// output words (+ the write-back ticket) the fused kernel accumulates into.
__global__ void copy_in_zero(uint32_t* __restrict__ dst, const uint32_t* __restrict__ src, int words,
                             uint32_t* __restrict__ zero, int zero_words) {
  asm volatile("griddepcontrol.launch_dependents;");   // the fused kernel may launch now (it waits)
  const int stride = gridDim.x * blockDim.x;
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < words; i += stride) dst[i] = src[i];
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < zero_words; i += stride) zero[i] = 0u;
}

// Word copy between device memory and mapped (page-locked) host memory: the small-problem
// host-buffer path moves its few kilobytes with kernels instead of copy-engine transfers.
__global__ void copy_words(uint32_t* __restrict__ dst, const uint32_t* __restrict__ src, int words) {
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < words; i += gridDim.x * blockDim.x) dst[i] = src[i];
}

// Sum G partial global copies into the output (one thread per bin, the paper's
// reduction kernel K13, L778-782).
__global__ void reduce_partials(const unsigned long long* __restrict__ part, int G, int nb,
                                OutSink out) {
  for (int k = blockIdx.x * blockDim.x + threadIdx.x; k < nb; k += gridDim.x * blockDim.x) {
    unsigned long long s = 0;
    for (int gi = 0; gi < G; ++gi) s += part[(size_t)gi * nb + k];
    if (out.n == 0) out.p[0][k] = s;      // overwrite: no zeroing of the output needed
    else if (s) out.add(k, s);
  }
  out.fence();
}

// ------------------------------------------------------------------------------------
// a11: Type-III pair matrix. Each thread owns 4 consecutive columns (registers) and
// walks kMatRows rows whose coordinates are warp-uniform loads; each row writes one
// float4 per thread with a streaming store: a warp writes 512 contiguous bytes.
// ------------------------------------------------------------------------------------
constexpr int kMatThreads = 256;
constexpr int kMatCols = kMatThreads * 4;  // 1024 columns per CTA
constexpr int kMatRows = 16;               // rows per CTA

template <int KTYPE, int D, bool VEC>
__global__ void __launch_bounds__(kMatThreads) pairmatrix_kernel(const float* __restrict__ soa, int n, int n_pad,
                                                                 int rb, int re, float cexp,
                                                                 float* __restrict__ out) {
  const int j0 = blockIdx.x * kMatCols + threadIdx.x * 4;
  const int r0 = rb + blockIdx.y * kMatRows;
  float pc[D][4];
#pragma unroll
  for (int c = 0; c < D; ++c) {
    const float4 v = *reinterpret_cast<const float4*>(soa + (long long)c * n_pad + j0);  // n_pad covers j0+3
    pc[c][0] = v.x; pc[c][1] = v.y; pc[c][2] = v.z; pc[c][3] = v.w;
  }
  const int rend = min(re, r0 + kMatRows);
  for (int i = r0; i < rend; ++i) {
    float a[D];
#pragma unroll
    for (int c = 0; c < D; ++c) a[c] = __ldg(soa + (long long)c * n_pad + i);
    float o[4];
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      float s = 0.f;
#pragma unroll
      for (int c = 0; c < D; ++c) {
        const float d = pc[c][q] - a[c];
        s = fmaf(d, d, s);
      }
      if (KTYPE == 0) o[q] = ex2_approx(cexp * s);  // exp(-gamma s) = 2^(-gamma log2(e) s)
      else if (KTYPE == 1) o[q] = s;
      else o[q] = sqrt_approx(s);
    }
    float* row = out + (size_t)(i - rb) * (size_t)n;
    if (VEC) {
      if (j0 < n) st_cs_v4(row + j0, o[0], o[1], o[2], o[3]);
    } else {
#pragma unroll
      for (int q = 0; q < 4; ++q)
        if (j0 + q < n) __stcs(row + j0 + q, o[q]);
    }
  }
}

}  // namespace tbs
