// tbs_api.cu — the C-ABI host library (libtbs.so): argument validation, output-stage
// selection, stream-ordered scratch, the work geometry, launches. Declared in
// include/tbs.h (which cites the paper passages defining each operation).
#include <cuda.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <chrono>
#include <atomic>
#include <cmath>
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <string>
#include <type_traits>
#include <vector>

#include "tbs.h"
#include "tbs_kernels.cuh"
#include "tbs_hd.cuh"
#include "tbs_hd2.cuh"
#include "tbs_knn.cuh"
#include "tbs_rdf.cuh"

using namespace tbs;
static_assert(kMaxPeers == TBS_MAX_PEERS, "peer sink size");

// Pair-engine configurations per output type: anchors/thread, partner chunk, CTAs/SM
// (A/B-tunable with -D at build time, see tools/build_ab.py).
// tensor-core pair matrix (tbs_hd2.cuh): operand ring stages / epilogue staging buffers for
// small d (<= 128: at most 2 k-blocks per tile) and large d
#ifndef TBS_HD2_RING_S
#define TBS_HD2_RING_S 4
#endif
#ifndef TBS_HD2_NSTG_S
#define TBS_HD2_NSTG_S 2
#endif
#ifndef TBS_HD2_RING_L
#define TBS_HD2_RING_L 4
#endif
#ifndef TBS_HD2_NSTG_L
#define TBS_HD2_NSTG_L 2
#endif
#ifndef TBS_SDH_KA
#define TBS_SDH_KA 8
#endif
#ifndef TBS_SDH_TP
#define TBS_SDH_TP 1024
#endif
#ifndef TBS_SDH_MINB
#define TBS_SDH_MINB 3
#endif
#ifndef TBS_PCF_KA
#define TBS_PCF_KA 8
#endif
#ifndef TBS_PCF_TP
#define TBS_PCF_TP 1024
#endif
#ifndef TBS_PCF_MINB
#define TBS_PCF_MINB 2
#endif
// kernel density (NEXT-2): 3 CTAs/SM measured +4.2 % over the 2PCF config (profiles/r02_sdh_config_ab.txt)
#ifndef TBS_KDE_KA
#define TBS_KDE_KA 8
#endif
#ifndef TBS_KDE_TP
#define TBS_KDE_TP 1024
#endif
#ifndef TBS_KDE_MINB
#define TBS_KDE_MINB 3
#endif
#ifndef TBS_LAT_KA
#define TBS_LAT_KA 8
#endif
#ifndef TBS_LAT_TP
#define TBS_LAT_TP 1024
#endif
#ifndef TBS_LAT_MINB
#define TBS_LAT_MINB 2
#endif
// Lattice fast variant (fp32 one-sided fix-up) compiled on its own: smaller register
// footprint than the kernel holding every exact-bucketing variant.
#ifndef TBS_LATF_KA
#define TBS_LATF_KA 8
#endif
#ifndef TBS_LATF_TP
#define TBS_LATF_TP 1024
#endif
#ifndef TBS_LATF_MINB
#define TBS_LATF_MINB 3
#endif
#define TBS_LATF_CFG TBS_LATF_KA, TBS_LATF_TP, TBS_LATF_MINB
#define TBS_SDH_CFG TBS_SDH_KA, TBS_SDH_TP, TBS_SDH_MINB
#define TBS_PCF_CFG TBS_PCF_KA, TBS_PCF_TP, TBS_PCF_MINB
#define TBS_LAT_CFG TBS_LAT_KA, TBS_LAT_TP, TBS_LAT_MINB
using SdhCfg = Cfg<TBS_SDH_CFG>;
using PcfCfg = Cfg<TBS_PCF_CFG>;
using KdeCfg = Cfg<TBS_KDE_KA, TBS_KDE_TP, TBS_KDE_MINB>;
using LatCfg = Cfg<TBS_LAT_CFG>;
using LatFastCfg = Cfg<TBS_LATF_CFG>;
// Small problems (fewer work items than ~2 per SM with the main configs): finer tiles so
// the grid covers the GPU (BASELINE configs[0], N = 4096, is launch/latency-bound).
#ifndef TBS_SMALL_TP
#define TBS_SMALL_TP 128
#endif
#ifndef TBS_SMALL_LOG2R
#define TBS_SMALL_LOG2R 5   // histogram replicas (2^x) of the small fused kernel
#endif
#ifndef TBS_SMALL_KA
#define TBS_SMALL_KA 2
#endif
#ifndef TBS_SMALL_MINB
#define TBS_SMALL_MINB 4
#endif
using SmallCfg = Cfg<TBS_SMALL_KA, TBS_SMALL_TP, TBS_SMALL_MINB>;
// Use the small-problem config when the main config yields fewer than this many items per SM.
int small_items_per_sm() {
  static const int v = [] { const char* e = getenv("TBS_SMALL_ITEMS"); return e ? atoi(e) : 16; }();
  return v;
}

namespace {

thread_local std::string g_err;
std::atomic<unsigned long long> g_launches{0};

int fail(int code, const char* fmt, ...) {
  char buf[512];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof(buf), fmt, ap);
  va_end(ap);
  g_err = buf;
  return code;
}

#define TBS_CUDA(call)                                                                        \
  do {                                                                                        \
    cudaError_t e_ = (call);                                                                  \
    if (e_ != cudaSuccess) return fail(TBS_ECUDA, "%s: %s (%s:%d)", #call, cudaGetErrorString(e_), __FILE__, __LINE__); \
  } while (0)

struct Device {
  int id = -1;
  int sms = 0;
  int smem_optin = 0;
};

int current_device(Device& d) {
  int dev;
  TBS_CUDA(cudaGetDevice(&dev));
  static thread_local Device cache;
  if (cache.id != dev) {
    cudaDeviceProp p;
    TBS_CUDA(cudaGetDeviceProperties(&p, dev));
    cache.id = dev;
    cache.sms = p.multiProcessorCount;
    cache.smem_optin = (int)p.sharedMemPerBlockOptin;
    // keep freed scratch cached in the stream-ordered pool (tbs_release() trims it)
    cudaMemPool_t pool;
    if (cudaDeviceGetDefaultMemPool(&pool, dev) == cudaSuccess) {
      unsigned long long thr = ~0ull;
      cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &thr);
    }
  }
  d = cache;
  return TBS_OK;
}

Geom make_geom(int64_t n, int64_t rb, int64_t re, int ta, int tp) {
  Geom g;
  g.n = (int)n;
  g.rb = (int)rb;
  g.re = (int)re;
  g.I0 = (int)(rb / ta);
  g.I1 = (int)((re + ta - 1) / ta);
  g.Mc = (int)((n + tp - 1) / tp);
  g.ratio = ta / tp;
  g.n_pad = (int)(((n + kPadAlign - 1) / kPadAlign) * kPadAlign);
  const long long I0 = g.I0, I1 = g.I1;
  g.items = (I1 - I0) * (long long)g.Mc - (long long)g.ratio * ((I1 * (I1 - 1) - I0 * (I0 - 1)) / 2);
  g.trace = nullptr;
  g.counter = nullptr;
  g.chunk = 1;
  return g;
}

int pad_rows(int64_t n) { return (int)(((n + kPadAlign - 1) / kPadAlign) * kPadAlign); }
int D_of(const tbs_args* a) { return a->dim <= 3 ? 3 : 4; }

// Persistent grid for a pair-kernel instantiation: SMs x resident CTAs (at most one CTA per item).
template <class Op, int D, class C, int VSET = 0x1F>
int launch_pair(const Device& dev, const float* soa, const tbs_args* a, const Op& op, const uint32_t* bbox,
                cudaStream_t st, cudaEvent_t eb, cudaEvent_t ee, bool first_launch_on_scratch = true,
                const OutSink& sink = OutSink{}, const TailPush& tail = TailPush{}) {
  // bbox may be nulled (TBS_FORCE_CLAMP); the 64-byte block always follows the SoA copy
  const uint32_t* bbox_block = reinterpret_cast<const uint32_t*>(soa + (size_t)D_of(a) * pad_rows(a->n));
  auto kern = pair_kernel<Op, D, C, VSET>;
  Geom g = make_geom(a->n, a->row_begin, a->row_end, C::TA, C::TP);
  // work queue head: the last u64 of the 64-byte bounding-box block (zeroed by the call's
  // memset; re-zeroed here for every further launch on the same scratch, e.g. bucket passes)
  g.counter = reinterpret_cast<unsigned long long*>(const_cast<uint32_t*>(bbox_block) + 14);
  if (!first_launch_on_scratch) TBS_CUDA(cudaMemsetAsync(g.counter, 0, sizeof(unsigned long long), st));
  const long long smem = ((op.smem_bytes() + 127) & ~127ll) + 2ll * D * C::TP * 4 + 16;
  if (smem > dev.smem_optin) return fail(TBS_EUNSUPPORTED, "pair kernel needs %lld B smem > %d", smem, dev.smem_optin);
  // per-instantiation cache of the attribute + occupancy query (host overhead of small calls)
  struct OccCache { int dev = -1; long long smem = -1; int occ = 0; };
  static thread_local OccCache cache;
  int occ = 0;
  if (cache.dev == dev.id && cache.smem == smem) {
    occ = cache.occ;
  } else {
    TBS_CUDA(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    TBS_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kern, kThreads, (size_t)smem));
    cache = OccCache{dev.id, smem, occ};
  }
  if (occ < 1) return fail(TBS_EUNSUPPORTED, "pair kernel cannot be resident (smem %lld)", smem);
  static const int occ_cap = [] {  // experiments only: TBS_OCC caps resident CTAs per SM
    const char* e = getenv("TBS_OCC");
    return e ? atoi(e) : 0;
  }();
  if (occ_cap > 0 && occ_cap < occ) occ = occ_cap;
  long long grid = (long long)dev.sms * occ;
  if (grid > g.items) grid = g.items;
  g.chunk = std::max<long long>(1, g.items / (grid * 200));   // ~200 grabs per CTA
  if (grid == g.items) g.chunk = 0;   // one item per CTA: static assignment, no queue round trips
  static const bool trace_on = getenv("TBS_TRACE") != nullptr;  // debug: CTA residency trace to stderr
  if (trace_on) TBS_CUDA(cudaMalloc(&g.trace, (size_t)grid * 3 * 8));
  if (eb) TBS_CUDA(cudaEventRecord(eb, st));
  kern<<<(unsigned)grid, kThreads, (size_t)smem, st>>>(soa, g, op, bbox, sink, tail);
  TBS_CUDA(cudaGetLastError());
  g_launches.fetch_add(1);
  if (ee) TBS_CUDA(cudaEventRecord(ee, st));
  if (trace_on) {
    std::vector<unsigned long long> t((size_t)grid * 3);
    TBS_CUDA(cudaStreamSynchronize(st));
    TBS_CUDA(cudaMemcpy(t.data(), g.trace, t.size() * 8, cudaMemcpyDeviceToHost));
    cudaFree(g.trace);
    unsigned long long t0 = ~0ull, t1 = 0;
    std::vector<int> per_sm(1024, 0);
    double dmin = 1e30, dmax = 0, dsum = 0;
    for (long long b = 0; b < grid; ++b) {
      t0 = std::min(t0, t[3 * b + 1]);
      t1 = std::max(t1, t[3 * b + 2]);
      per_sm[t[3 * b] & 1023]++;
      const double d = (double)(t[3 * b + 2] - t[3 * b + 1]);
      dmin = std::min(dmin, d); dmax = std::max(dmax, d); dsum += d;
    }
    int mx = 0, mn = 1 << 30;
    for (int k = 0; k < dev.sms; ++k) { mx = std::max(mx, per_sm[k]); mn = std::min(mn, per_sm[k]); }
    double late = 0;  // latest CTA start relative to kernel start
    for (long long b = 0; b < grid; ++b) late = std::max(late, (double)(t[3 * b + 1] - t0));
    fprintf(stderr, "[tbs trace] grid %lld occ %d: CTAs/SM %d..%d, CTA time min %.3f avg %.3f max %.3f ms, "
            "span %.3f ms, latest start %.3f ms\n", grid, occ, mn, mx, dmin * 1e-6, dsum / grid * 1e-6, dmax * 1e-6,
            (t1 - t0) * 1e-6, late * 1e-6);
  }
  return TBS_OK;
}

// Small problems (fewer items than small_items_per_sm() per SM, n <= kSmallLoad): the fused
// one-item-per-CTA kernel reading the caller's AoS points (no loader launch, no SoA scratch).
bool small_fused(const Device& dev, const tbs_args* a) {
  if (a->n > kSmallLoad || (a->flags & TBS_VALIDATE)) return false;
  return make_geom(a->n, a->row_begin, a->row_end, SdhCfg::TA, SdhCfg::TP).items <
         (long long)small_items_per_sm() * dev.sms;
}

// A host-buffer call's request to the small fused path (thread-local, set by run_simple around
// its call): the output and ticket are already zeroed; the kernel's last CTA writes the result
// to mapped host memory. `taken` reports whether the path consumed it.
struct SmallWriteBack {
  WriteBack wb;
  bool active = false, taken = false;
};
SmallWriteBack& small_wb() {
  static thread_local SmallWriteBack w;
  return w;
}

// TBS_SMALL_PDL=0 (A/B): launch the small fused kernel after the copy kernel without
// programmatic dependent launch.
bool small_pdl() {
  static const bool v = [] { const char* e = getenv("TBS_SMALL_PDL"); return !(e && atoi(e) == 0); }();
  return v;
}

template <class Op, int D, int V>
int launch_small(const Device& dev, const tbs_args* a, const Op& op, cudaStream_t st, cudaEvent_t eb, cudaEvent_t ee,
                 const OutSink& sink) {
  using C = SmallCfg;
  auto kern = pair_kernel_small<Op, D, C, V>;
  const Geom g = make_geom(a->n, a->row_begin, a->row_end, C::TA, C::TP);
  const long long smem = ((op.smem_bytes() + 127) & ~127ll) + (long long)D * C::TP * 4 + 16;
  if (smem > dev.smem_optin) return fail(TBS_EUNSUPPORTED, "small pair kernel needs %lld B smem", smem);
  struct AttrCache { int dev = -1; long long smem = -1; };
  static thread_local AttrCache cache;
  if (cache.dev != dev.id || cache.smem < smem) {
    TBS_CUDA(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    cache = AttrCache{dev.id, smem};
  }
  if (eb) TBS_CUDA(cudaEventRecord(eb, st));
  WriteBack wb{};
  if (small_wb().active) {
    wb = small_wb().wb;
    small_wb().taken = true;
  }
  if (wb.dst != nullptr && small_pdl()) {
    // after the host-buffer path's copy kernel: programmatic dependent launch (the grid starts
    // early and waits in-kernel for the copy; griddepcontrol.wait)
    cudaLaunchConfig_t cfg{};
    cfg.gridDim = dim3((unsigned)g.items);
    cfg.blockDim = dim3(kThreads);
    cfg.dynamicSmemBytes = (size_t)smem;
    cfg.stream = st;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    TBS_CUDA(cudaLaunchKernelEx(&cfg, kern, a->points, a->dim, g, op, sink, wb));
  } else {
    kern<<<(unsigned)g.items, kThreads, (size_t)smem, st>>>(a->points, a->dim, g, op, sink, wb);
  }
  TBS_CUDA(cudaGetLastError());
  g_launches.fetch_add(1);
  if (ee) TBS_CUDA(cudaEventRecord(ee, st));
  return TBS_OK;
}

// peer_words: the output words of this operation (SDH nb, 2PCF 1) under TBS_OUT_PEERS; 0 = the
// operation does not support the fused combine.
int validate_common(const tbs_args* a, long long peer_words = 0) {
  if (!a) return fail(TBS_EINVAL, "args is NULL");
  if (a->flags & TBS_OUT_PEERS) {
    if (peer_words == 0) return fail(TBS_EUNSUPPORTED, "TBS_OUT_PEERS: SDH and 2PCF only");
    if (a->n_out_peers < 1 || a->n_out_peers > kMaxPeers || !a->out_peers)
      return fail(TBS_EINVAL, "TBS_OUT_PEERS needs 1..%d out_peers", kMaxPeers);
    for (int w = 0; w < a->n_out_peers; ++w)
      if (!a->out_peers[w]) return fail(TBS_EINVAL, "out_peers[%d] is NULL", w);
    if (a->out_peer_words != peer_words)
      return fail(TBS_EINVAL, "TBS_OUT_PEERS: out_peer_words = %lld, this call writes %lld words",
                  (long long)a->out_peer_words, peer_words);
  }
  if (a->n < 0 || a->n > TBS_MAX_N) return fail(TBS_EINVAL, "n = %lld outside [0, 2^30]", (long long)a->n);
  if (a->dim < 1 || a->dim > 4) return fail(TBS_EINVAL, "dim = %d outside [1, 4]", a->dim);
  if (a->row_begin < 0 || a->row_end < a->row_begin || a->row_end > a->n)
    return fail(TBS_EINVAL, "row range [%lld, %lld) outside [0, %lld]", (long long)a->row_begin,
                (long long)a->row_end, (long long)a->n);
  if (a->n >= 2 && !a->points) return fail(TBS_EINVAL, "points is NULL");
  return TBS_OK;
}

void release_soa(float* soa, cudaStream_t st) {
  if (soa) cudaFreeAsync(soa, st);
}

// SoA copy of the points in stream-ordered scratch; the loader also zeroes `zero` words.
// The allocation holds SoA [D][n_pad] followed by the 2D+1 bounding-box words.
int load_points(const tbs_args* a, int D, int n_pad, float** soa, unsigned long long* zero, long long zero_words,
                cudaStream_t st, uint32_t** bbox, float pad = 0.0f) {
  const size_t soa_bytes = (size_t)D * n_pad * sizeof(float);
  TBS_CUDA(cudaMallocAsync((void**)soa, soa_bytes + 64, st));
  *bbox = reinterpret_cast<uint32_t*>(reinterpret_cast<unsigned char*>(*soa) + soa_bytes);
  // Small problems: one 1024-thread CTA writes the whole bounding-box block itself (no memset
  // launch before it: the small-problem path is latency-bound, BASELINE configs[0]).
  if (n_pad <= kSmallLoad && zero_words <= (1 << 16)) {
    if (D == 3)
      soa_loader_small<3><<<1, 1024, 0, st>>>(a->points, (int)a->n, a->dim, n_pad, pad, *soa, zero, (int)zero_words, *bbox);
    else
      soa_loader_small<4><<<1, 1024, 0, st>>>(a->points, (int)a->n, a->dim, n_pad, pad, *soa, zero, (int)zero_words, *bbox);
  } else {
    TBS_CUDA(cudaMemsetAsync(*bbox, 0, 64, st));
    const int threads = 256;
    long long blocks = std::min<long long>((n_pad + threads - 1) / threads, 148ll * 8);
    blocks = std::max<long long>(blocks, 1);
    soa_loader<<<(unsigned)blocks, threads, 0, st>>>(a->points, (int)a->n, a->dim, n_pad, D, pad, *soa, zero,
                                                     zero_words, *bbox);
  }
  TBS_CUDA(cudaGetLastError());
  g_launches.fetch_add(1);
  return TBS_OK;
}

// TBS_VALIDATE (debug): wait for the loader and check what it recorded in the
// bounding-box block: non-finite coordinates; under the exact-lattice contract also non-integer
// coordinates and a spread whose squared pair distances could reach 2^24.
int validate_points(const tbs_args* a, const uint32_t* bbox, int D, bool lattice, cudaStream_t st) {
  if (!(a->flags & TBS_VALIDATE) || a->n < 1) return TBS_OK;
  uint32_t h[9] = {0};
  TBS_CUDA(cudaMemcpyAsync(h, bbox, (size_t)(2 * D + 1) * 4, cudaMemcpyDeviceToHost, st));
  TBS_CUDA(cudaStreamSynchronize(st));
  if (h[2 * D] & 1u) return fail(TBS_EINVAL, "TBS_VALIDATE: non-finite coordinate");
  if (lattice) {
    if (h[2 * D] & 2u) return fail(TBS_EINVAL, "TBS_VALIDATE: TBS_EXACT_LATTICE needs integer-valued coordinates");
    auto ord2f_h = [](uint32_t o) {
      const uint32_t b = (o & 0x80000000u) ? (o & 0x7fffffffu) : ~o;
      float f;
      memcpy(&f, &b, 4);
      return (double)f;
    };
    double s = 0.0;
    for (int c = 0; c < D; ++c) {
      const double e = ord2f_h(h[D + c]) - ord2f_h(~h[c]);
      s += e * e;
    }
    if (s >= 16777216.0)
      return fail(TBS_EINVAL, "TBS_VALIDATE: TBS_EXACT_LATTICE needs every squared pair distance < 2^24 "
                  "(bounding-box bound %.0f)", s);
  }
  return TBS_OK;
}

// Output sink of the kernels of a Type-I/II call: one device buffer (the caller's output, or
// under TBS_OUT_PEERS the call's local accumulator).
OutSink local_sink(unsigned long long* buf) {
  OutSink o{};
  o.n = 0;
  o.p[0] = buf;
  return o;
}

OutSink peer_sink(const tbs_args* a) {
  OutSink o{};
  o.n = a->n_out_peers;
  for (int w = 0; w < o.n; ++w) o.p[w] = reinterpret_cast<unsigned long long*>(a->out_peers[w]);
  return o;
}

// TBS_OUT_PEERS in the pair kernel's tail (single-launch output stages): the last CTA pushes
// the local accumulator `acc` (words u64) into every rank's buffer; `ticket` is a zeroed u32.
TailPush tail_push(const tbs_args* a, const unsigned long long* acc, int words, uint32_t* ticket) {
  TailPush t{};
  t.peers = peer_sink(a);
  t.acc = acc;
  t.ticket = ticket;
  t.words = words;
  return t;
}

// TBS_OUT_PEERS, second stage as its own launch (multi-launch output stages: bucket-range
// passes, global partials + reduce, the small fused path): add the local accumulator into
// every rank's buffer.
int push_to_peers(const tbs_args* a, const unsigned long long* acc, int words, cudaStream_t st) {
  const OutSink o = peer_sink(a);
  push_peers<<<(words + 255) / 256, 256, 0, st>>>(acc, words, o);
  TBS_CUDA(cudaGetLastError());
  g_launches.fetch_add(1);
  return TBS_OK;
}

// Decompose a dyadic width w = m * 2^-j (m odd or j = 0). Returns false if not dyadic.
bool dyadic(float w, long long& m, int& j) {
  double x = (double)w;
  for (j = 0; j <= 19; ++j) {
    double v = std::ldexp(x, j);
    if (v == std::floor(v) && v >= 1.0 && v < 2147483648.0) {
      m = (long long)v;
      return true;
    }
  }
  return false;
}

struct SdhPlan {
  bool lattice, global;
  int log2r;
  int passes = 1;       // > 1: R = 1 bucket-range passes
  int pass_rows = 0;    // buckets per pass
};

// Lattice mode: the fast variants 4 and 0 (their own instantiation, LatFastCfg) and the
// exact general variants 1-3 (LatCfg) are two launches; the one whose variant the bounding box does
// not select exits at once (the work-queue counter is untouched by it).
// (Both launches carry the fused-combine tail: only the working one takes tickets.)
template <class Op, int D, class C, bool LAT>
int launch_sdh(const Device& dev, const float* soa, const tbs_args* g, const Op& op, const uint32_t* bbox,
               cudaStream_t st, cudaEvent_t eb, cudaEvent_t ee, const OutSink& sink, const TailPush& tail) {
  if constexpr (!LAT) {
    return launch_pair<Op, D, C>(dev, soa, g, op, bbox, st, eb, ee, true, sink, tail);
  } else {
    int rc = launch_pair<Op, D, LatFastCfg, 0x11>(dev, soa, g, op, bbox, st, eb, nullptr, true, sink, tail);
    if (rc) return rc;
    return launch_pair<Op, D, C, 0xE>(dev, soa, g, op, bbox, st, nullptr, ee, true, sink, tail);
  }
}

template <int D, bool LAT>
int sdh_dispatch(const Device& dev, const SdhPlan& pl, const float* soa, const uint32_t* bbox, const tbs_args* g, float w,
                 long long m, int j, int nb, const OutSink& hist, unsigned long long* part, int G, cudaStream_t st,
                 cudaEvent_t eb, cudaEvent_t ee, const TailPush& tail, bool& pushed) {
  pushed = false;   // set when a single-launch output stage carried the fused-combine tail
  if (pl.global) {
    SdhGlobalOp<LAT> op{};
    op.nb = nb;
    op.inv_w = (float)(1.0 / (double)w);
    op.scale = (float)std::ldexp(1.0 / (double)m, j);
    op.m = (int)m;
    op.sh = 2 * j;
    op.G = G;
    op.part = part;
    int rc = launch_pair<SdhGlobalOp<LAT>, D, SdhCfg>(dev, soa, g, op, bbox, st, eb, ee);
    if (rc) return rc;
    reduce_partials<<<(nb + 255) / 256, 256, 0, st>>>(part, G, nb, hist);
    TBS_CUDA(cudaGetLastError());
    g_launches.fetch_add(1);
    return TBS_OK;
  }
  auto fill = [&](auto& op, int R, long long ka_tp) {
    op.nb = nb;
    op.rows = nb + kGuard;
    op.inv_w = (float)(1.0 / (double)w);
    op.scale = (float)std::ldexp(1.0 / (double)m, j);
    op.scale_up = std::nextafter((float)(std::ldexp(1.0 / (double)m, j) * (1.0 + std::ldexp(1.0, -17))), INFINITY);
    op.scale_b = std::nextafter((float)(std::ldexp(1.0 / (double)m, j) * (1.0 + std::ldexp(1.0, -19))), INFINITY);
    op.mj = (float)std::ldexp((double)m, -j);
    op.m = (int)m;
    op.sh = 2 * j;
    // per item, a replica receives at most (32/R) lanes x kWarps x KA x TP increments
    if (LAT) ka_tp = std::max<long long>(ka_tp, (long long)LatFastCfg::KA * LatFastCfg::TP);
    const long long per_item = (long long)(32 / R) * kWarps * ka_tp;
    op.flush_every = (int)std::max<long long>(1, (0xffffffffll / per_item) - 1);
  };
  using C = typename std::conditional<LAT, LatCfg, SdhCfg>::type;
  const bool small =
      !LAT && make_geom(g->n, g->row_begin, g->row_end, C::TA, C::TP).items < (long long)small_items_per_sm() * dev.sms;
  if (pl.passes > 1) {
    int rc = TBS_OK;
    for (int p = 0; p < pl.passes && rc == TBS_OK; ++p) {
      SdhSmemOp<0, LAT, true> op{};
      fill(op, 1, (long long)C::KA * C::TP);
      op.klo = p * pl.pass_rows;
      const bool last = p + 1 == pl.passes;
      op.rows = last ? (nb - op.klo) + (LAT ? 0 : kGuard) : pl.pass_rows;
      rc = launch_pair<SdhSmemOp<0, LAT, true>, D, C>(dev, soa, g, op, bbox, st, p == 0 ? eb : nullptr,
                                                       last ? ee : nullptr, p == 0, hist);
    }
    return rc;
  }
  switch (pl.log2r) {
    case 5: {
      SdhSmemOp<5, LAT> op{};
      if constexpr (!LAT) {   // (lattice mode never takes the small-problem config)
        if (small) {
          fill(op, 32, (long long)SmallCfg::KA * SmallCfg::TP);
          pushed = tail.words > 0;
          return launch_pair<SdhSmemOp<5, LAT>, D, SmallCfg>(dev, soa, g, op, bbox, st, eb, ee, true, hist, tail);
        }
      }
      fill(op, 32, (long long)C::KA * C::TP);
      pushed = tail.words > 0;
      return launch_sdh<SdhSmemOp<5, LAT>, D, C, LAT>(dev, soa, g, op, bbox, st, eb, ee, hist, tail);
    }
    case 4: {
      SdhSmemOp<4, LAT> op{};
      fill(op, 16, (long long)C::KA * C::TP);
      pushed = tail.words > 0;
      return launch_sdh<SdhSmemOp<4, LAT>, D, C, LAT>(dev, soa, g, op, bbox, st, eb, ee, hist, tail);
    }
    case 3: {
      SdhSmemOp<3, LAT> op{};
      fill(op, 8, (long long)C::KA * C::TP);
      pushed = tail.words > 0;
      return launch_sdh<SdhSmemOp<3, LAT>, D, C, LAT>(dev, soa, g, op, bbox, st, eb, ee, hist, tail);
    }
    case 2: {
      SdhSmemOp<2, LAT> op{};
      fill(op, 4, (long long)C::KA * C::TP);
      pushed = tail.words > 0;
      return launch_sdh<SdhSmemOp<2, LAT>, D, C, LAT>(dev, soa, g, op, bbox, st, eb, ee, hist, tail);
    }
    case 1: {
      SdhSmemOp<1, LAT> op{};
      fill(op, 2, (long long)C::KA * C::TP);
      pushed = tail.words > 0;
      return launch_sdh<SdhSmemOp<1, LAT>, D, C, LAT>(dev, soa, g, op, bbox, st, eb, ee, hist, tail);
    }
    default: {
      SdhSmemOp<0, LAT> op{};
      fill(op, 1, (long long)C::KA * C::TP);
      pushed = tail.words > 0;
      return launch_sdh<SdhSmemOp<0, LAT>, D, C, LAT>(dev, soa, g, op, bbox, st, eb, ee, hist, tail);
    }
  }
}

int sdh_impl(const tbs_args* a, float w, int nb, uint64_t* hist) {
  int rc = validate_common(a, nb);
  if (rc) return rc;
  if (nb < 1 || nb > TBS_MAX_BUCKETS) return fail(TBS_EINVAL, "nbuckets = %d outside [1, 2^24]", nb);
  if (!(w > 0.f) || !std::isfinite(w)) return fail(TBS_EINVAL, "bucket_width must be finite and > 0");
  const bool peers = (a->flags & TBS_OUT_PEERS) != 0;
  if (!hist && !peers) return fail(TBS_EINVAL, "hist is NULL");
  const bool lattice = (a->flags & TBS_EXACT_LATTICE) != 0;
  long long m = 1;
  int j = 0;
  if (lattice) {
    if (!dyadic(w, m, j)) return fail(TBS_EINVAL, "TBS_EXACT_LATTICE needs bucket_width = m * 2^-j, j <= 19");
    if ((long long)(nb + 1) * m >= (1ll << 31)) return fail(TBS_EINVAL, "TBS_EXACT_LATTICE needs (nb+1)*m < 2^31");
  }
  Device dev;
  if ((rc = current_device(dev))) return rc;
  cudaStream_t st = (cudaStream_t)a->stream;
  auto* h = reinterpret_cast<unsigned long long*>(hist);
  if (a->n < 2 || a->row_begin >= a->row_end) {
    if (!peers) TBS_CUDA(cudaMemsetAsync(h, 0, (size_t)nb * 8, st));   // (fused combine: adds nothing)
    return TBS_OK;
  }
  unsigned long long* acc = nullptr;   // TBS_OUT_PEERS: this rank's partial, pushed to every rank at the end
  if (peers) {
    TBS_CUDA(cudaMallocAsync((void**)&acc, (size_t)nb * 8, st));
    h = acc;
  }
  const OutSink sink = local_sink(h);
  // Output-stage plan: lane-private copies (R = 32) while they fit a 96 KB budget (two CTAs
  // per SM), then 4 replicas, then one copy per CTA; beyond that, global partial copies.
  SdhPlan pl{lattice, false, 5};
  const long long part_budget = std::min<long long>(96 * 1024, dev.smem_optin - 2ll * 4 * SdhCfg::TP * 4 - 256);
  const long long one_copy_budget = dev.smem_optin - 2ll * 4 * SdhCfg::TP * 4 - 256;
  // Measured on B200 (tools/ab_r.sh, N=1M): the most replicas that fit win even at one CTA
  // per SM, except that R = 32 is only worth it while it leaves room for 2+ CTAs.
  const long long rows = nb + kGuard + 1;   // + the trash row of masked pairs
  if (rows * 32 * 4 <= part_budget) pl.log2r = 5;
  else if (rows * 16 * 4 <= one_copy_budget) pl.log2r = 4;
  else if (rows * 8 * 4 <= one_copy_budget) pl.log2r = 3;
  else if (rows * 4 * 4 <= one_copy_budget) pl.log2r = 2;
  else if (rows * 2 * 4 <= one_copy_budget) pl.log2r = 1;
  else if (rows * 4 <= one_copy_budget) pl.log2r = 0;
  else {
    // beyond one copy: up to 8 bucket-range passes with one copy (each pass ~2.5e12 pairs/s
    // vs ~0.2e12 for L2 atomics), else the partially privatised global histogram
    const int per_pass = (int)(one_copy_budget / 4) - kGuard - 1;
    const int passes = (nb + per_pass - 1) / per_pass;
    if (passes <= 8) {
      pl.log2r = 0;
      pl.passes = passes;
      pl.pass_rows = per_pass;
    } else {
      pl.global = true;
    }
  }
  static const int r_env = [] { const char* e = getenv("TBS_LOG2R"); return e ? atoi(e) : -1; }();  // experiments
  if (r_env >= 0 && !pl.global && pl.passes == 1 && rows * (4ll << r_env) <= one_copy_budget)
    pl.log2r = r_env;
  if (a->flags & TBS_HIST_FORCE_LANE) {
    if (rows * 32 * 4 > one_copy_budget) return fail(TBS_EUNSUPPORTED, "FORCE_LANE: nb too large for smem");
    pl = SdhPlan{lattice, false, 5};
  }
  if (a->flags & TBS_HIST_FORCE_CTA) {
    if (rows * 4 > one_copy_budget) return fail(TBS_EUNSUPPORTED, "FORCE_CTA: nb too large for smem");
    pl = SdhPlan{lattice, false, 0};
  }
  if (a->flags & TBS_HIST_FORCE_PASSES) {   // bucket-range passes even when one copy fits (tests)
    pl = SdhPlan{lattice, false, 0};
    pl.pass_rows = std::max(1, (nb + 2) / 3);
    pl.passes = (nb + pl.pass_rows - 1) / pl.pass_rows;
  }
  if (a->flags & TBS_HIST_FORCE_GLOBAL) pl = SdhPlan{lattice, true, 0};

  const int D = a->dim <= 3 ? 3 : 4;
  if (!lattice && !pl.global && pl.passes == 1 && pl.log2r == 5 && small_fused(dev, a)) {
    // small problem: zero the output, one fused launch (clamp variant: no bounding box)
    using SOp = SdhSmemOp<TBS_SMALL_LOG2R, false>;
    SOp op{};
    op.nb = nb;
    op.rows = nb + kGuard;
    op.inv_w = (float)(1.0 / (double)w);
    op.flush_every = (int)std::max<long long>(
        1, 0xffffffffll / ((long long)(32 >> TBS_SMALL_LOG2R) * kWarps * SmallCfg::KA * SmallCfg::TP) - 1);
    if (!small_wb().active || peers) TBS_CUDA(cudaMemsetAsync(h, 0, (size_t)nb * 8, st));
    cudaEvent_t eb = (cudaEvent_t)a->ev_begin, ee = (cudaEvent_t)a->ev_end;
    rc = D == 3 ? launch_small<SOp, 3, 1>(dev, a, op, st, eb, ee, sink)
                : launch_small<SOp, 4, 1>(dev, a, op, st, eb, ee, sink);
    if (!rc && peers) rc = push_to_peers(a, acc, nb, st);
    if (acc) cudaFreeAsync(acc, st);
    return rc;
  }
  const int n_pad = pad_rows(a->n);
  int G = 0;
  unsigned long long* part = nullptr;
  long long zero_words = 0;
  if (pl.global) {
    G = std::min(dev.sms, 64);
    TBS_CUDA(cudaMallocAsync((void**)&part, (size_t)G * nb * 8, st));
    zero_words = (long long)G * nb;
  }
  float* soa = nullptr;
  // Smem modes accumulate into hist (or the fused combine's local accumulator): the loader
  // zeroes it. Global mode zeroes the partials (the reduce kernel overwrites hist).
  uint32_t* bbox = nullptr;
  rc = load_points(a, D, n_pad, &soa, pl.global ? part : h, pl.global ? zero_words : nb, st, &bbox);
  if (!rc) rc = validate_points(a, bbox, D, lattice, st);
  // fused combine in the pair kernel's tail: ticket = the zeroed spare word 12 of the box block
  const TailPush tail = peers && !rc ? tail_push(a, acc, nb, bbox + 12) : TailPush{};
  if (a->flags & TBS_FORCE_CLAMP) bbox = nullptr;
  bool pushed = false;
  if (!rc) {
    cudaEvent_t eb = (cudaEvent_t)a->ev_begin, ee = (cudaEvent_t)a->ev_end;
    if (D == 3) rc = lattice ? sdh_dispatch<3, true>(dev, pl, soa, bbox, a, w, m, j, nb, sink, part, G, st, eb, ee, tail, pushed)
                             : sdh_dispatch<3, false>(dev, pl, soa, bbox, a, w, m, j, nb, sink, part, G, st, eb, ee, tail, pushed);
    else rc = lattice ? sdh_dispatch<4, true>(dev, pl, soa, bbox, a, w, m, j, nb, sink, part, G, st, eb, ee, tail, pushed)
                      : sdh_dispatch<4, false>(dev, pl, soa, bbox, a, w, m, j, nb, sink, part, G, st, eb, ee, tail, pushed);
  }
  if (!rc && peers && !pushed) rc = push_to_peers(a, acc, nb, st);
  release_soa(soa, st);
  if (part) cudaFreeAsync(part, st);
  if (acc) cudaFreeAsync(acc, st);
  return rc;
}

int pcf_impl(const tbs_args* a, float r, uint64_t* count) {
  int rc = validate_common(a, 1);
  if (rc) return rc;
  if (!(r >= 0.f) || std::isinf(r)) return fail(TBS_EINVAL, "radius must be finite and >= 0");
  const bool peers = (a->flags & TBS_OUT_PEERS) != 0;
  if (!count && !peers) return fail(TBS_EINVAL, "count is NULL");
  Device dev;
  if ((rc = current_device(dev))) return rc;
  cudaStream_t st = (cudaStream_t)a->stream;
  auto* c = reinterpret_cast<unsigned long long*>(count);
  if (a->n < 2 || a->row_begin >= a->row_end) {
    if (!peers) TBS_CUDA(cudaMemsetAsync(c, 0, 8, st));
    return TBS_OK;
  }
  const int D = a->dim <= 3 ? 3 : 4;
  if (!peers && small_fused(dev, a)) {
    PcfOp op{};
    op.r2 = (float)((double)r * (double)r);
    if (!small_wb().active) TBS_CUDA(cudaMemsetAsync(c, 0, 8, st));
    cudaEvent_t eb = (cudaEvent_t)a->ev_begin, ee = (cudaEvent_t)a->ev_end;
    return D == 3 ? launch_small<PcfOp, 3, 0>(dev, a, op, st, eb, ee, local_sink(c))
                  : launch_small<PcfOp, 4, 0>(dev, a, op, st, eb, ee, local_sink(c));
  }
  float* soa = nullptr;
  uint32_t* bbox = nullptr;
  rc = load_points(a, D, pad_rows(a->n), &soa, peers ? nullptr : c, peers ? 0 : 1, st, &bbox);
  if (!rc) rc = validate_points(a, bbox, D, false, st);
  // TBS_OUT_PEERS: the local accumulator is the zeroed spare u64 at byte 40 of the bounding-box
  // block (words 0..2D are the box, 12 the fused combine's ticket, 14-15 the work counter)
  unsigned long long* acc = peers ? reinterpret_cast<unsigned long long*>(bbox + 10) : c;
  if (!rc) {
    PcfOp op{};
    op.r2 = (float)((double)r * (double)r);
    const OutSink sink = local_sink(acc);
    // fused combine in the pair kernel's tail (ticket: the zeroed spare word 12 of the box block)
    const TailPush tail = peers ? tail_push(a, acc, 1, bbox + 12) : TailPush{};
    cudaEvent_t eb = (cudaEvent_t)a->ev_begin, ee = (cudaEvent_t)a->ev_end;
    const bool small =
        make_geom(a->n, a->row_begin, a->row_end, PcfCfg::TA, PcfCfg::TP).items < (long long)small_items_per_sm() * dev.sms;
    if (small)
      rc = D == 3 ? launch_pair<PcfOp, 3, SmallCfg>(dev, soa, a, op, bbox, st, eb, ee, true, sink, tail)
                  : launch_pair<PcfOp, 4, SmallCfg>(dev, soa, a, op, bbox, st, eb, ee, true, sink, tail);
    else
      rc = D == 3 ? launch_pair<PcfOp, 3, PcfCfg>(dev, soa, a, op, bbox, st, eb, ee, true, sink, tail)
                  : launch_pair<PcfOp, 4, PcfCfg>(dev, soa, a, op, bbox, st, eb, ee, true, sink, tail);
  }
  release_soa(soa, st);
  return rc;
}

int kde_impl(const tbs_args* a, float gamma, double* sum) {
  int rc = validate_common(a);
  if (rc) return rc;
  if (!std::isfinite(gamma)) return fail(TBS_EINVAL, "gamma must be finite");
  if (!sum) return fail(TBS_EINVAL, "sum is NULL");
  Device dev;
  if ((rc = current_device(dev))) return rc;
  cudaStream_t st = (cudaStream_t)a->stream;
  if (a->n < 2 || a->row_begin >= a->row_end) {
    TBS_CUDA(cudaMemsetAsync(sum, 0, 8, st));
    return TBS_OK;
  }
  const int D = a->dim <= 3 ? 3 : 4;
  if (small_fused(dev, a)) {
    KdeOp op{};
    op.c = (float)(-(double)gamma * 1.4426950408889634);
    op.sum = sum;
    if (!small_wb().active) TBS_CUDA(cudaMemsetAsync(sum, 0, 8, st));
    cudaEvent_t eb = (cudaEvent_t)a->ev_begin, ee = (cudaEvent_t)a->ev_end;
    return D == 3 ? launch_small<KdeOp, 3, 0>(dev, a, op, st, eb, ee, OutSink{})
                  : launch_small<KdeOp, 4, 0>(dev, a, op, st, eb, ee, OutSink{});
  }
  float* soa = nullptr;
  uint32_t* bbox = nullptr;
  rc = load_points(a, D, pad_rows(a->n), &soa, reinterpret_cast<unsigned long long*>(sum), 1, st, &bbox);
  if (!rc) rc = validate_points(a, bbox, D, false, st);
  if (!rc) {
    KdeOp op{};
    op.c = (float)(-(double)gamma * 1.4426950408889634);
    op.sum = sum;
    cudaEvent_t eb = (cudaEvent_t)a->ev_begin, ee = (cudaEvent_t)a->ev_end;
    const bool small =
        make_geom(a->n, a->row_begin, a->row_end, PcfCfg::TA, PcfCfg::TP).items < (long long)small_items_per_sm() * dev.sms;
    if (small)
      rc = D == 3 ? launch_pair<KdeOp, 3, SmallCfg>(dev, soa, a, op, bbox, st, eb, ee)
                  : launch_pair<KdeOp, 4, SmallCfg>(dev, soa, a, op, bbox, st, eb, ee);
    else
      rc = D == 3 ? launch_pair<KdeOp, 3, KdeCfg>(dev, soa, a, op, bbox, st, eb, ee)
                  : launch_pair<KdeOp, 4, KdeCfg>(dev, soa, a, op, bbox, st, eb, ee);
  }
  release_soa(soa, st);
  return rc;
}

// ---- NEXT-1: radial distribution function (reading R6) ------------------------------------
int rdf_normalize(const uint64_t* hist, int nb, int dim, float w, double pairs, double volume, double* g,
                  cudaStream_t st) {
  const int threads = 256;
  const int blocks = std::min((nb + threads - 1) / threads, 1024);
  rdf_kernel<<<blocks, threads, 0, st>>>(reinterpret_cast<const unsigned long long*>(hist), nb, dim, (double)w, pairs,
                                         volume, g);
  TBS_CUDA(cudaGetLastError());
  g_launches.fetch_add(1);
  return TBS_OK;
}

int rdf_args_ok(int nb, int dim, float w, double volume, const double* g) {
  if (nb < 1 || nb >= TBS_MAX_BUCKETS) return fail(TBS_EINVAL, "nbuckets = %d outside [1, 2^24)", nb);
  if (dim < 1 || dim > 4) return fail(TBS_EINVAL, "dim = %d outside [1, 4]", dim);
  if (!(w > 0.f) || !std::isfinite(w)) return fail(TBS_EINVAL, "bucket_width must be finite and > 0");
  if (!(volume > 0.0) || !std::isfinite(volume)) return fail(TBS_EINVAL, "volume must be finite and > 0");
  if (!g) return fail(TBS_EINVAL, "g is NULL");
  return TBS_OK;
}

int rdf_impl(const tbs_args* a, float w, int nb, double volume, double* g) {
  int rc = validate_common(a);
  if (rc) return rc;
  if ((rc = rdf_args_ok(nb, a->dim, w, volume, g))) return rc;
  cudaStream_t st = (cudaStream_t)a->stream;
  uint64_t* h = nullptr;
  TBS_CUDA(cudaMallocAsync((void**)&h, (size_t)(nb + 1) * 8, st));
  rc = sdh_impl(a, w, nb + 1, h);   // bucket nb takes every d >= nb w (the clamp): not a shell
  if (!rc) {
    const double rows = (double)(a->row_end - a->row_begin);
    const double pairs = rows * (double)(2 * a->n - a->row_begin - a->row_end - 1) / 2.0;
    rc = rdf_normalize(h, nb, a->dim, w, pairs, volume, g, st);
  }
  cudaFreeAsync(h, st);
  return rc;
}

template <int KT, int D>
int matrix_launch(const tbs_args* a, const float* soa, int n_pad, float cexp, float* out, cudaStream_t st) {
  const int n = (int)a->n;
  dim3 grid((unsigned)((n + kMatCols - 1) / kMatCols), (unsigned)((a->row_end - a->row_begin + kMatRows - 1) / kMatRows));
  if (grid.y > 2147483647u) return fail(TBS_EUNSUPPORTED, "too many rows");
  cudaEvent_t eb = (cudaEvent_t)a->ev_begin, ee = (cudaEvent_t)a->ev_end;
  if (eb) TBS_CUDA(cudaEventRecord(eb, st));
  if (n % 4 == 0)
    pairmatrix_kernel<KT, D, true><<<grid, kMatThreads, 0, st>>>(soa, n, n_pad, (int)a->row_begin, (int)a->row_end, cexp, out);
  else
    pairmatrix_kernel<KT, D, false><<<grid, kMatThreads, 0, st>>>(soa, n, n_pad, (int)a->row_begin, (int)a->row_end, cexp, out);
  TBS_CUDA(cudaGetLastError());
  g_launches.fetch_add(1);
  if (ee) TBS_CUDA(cudaEventRecord(ee, st));
  return TBS_OK;
}

int pairmatrix_impl(const tbs_args* a, tbs_kernel k, float* out) {
  int rc = validate_common(a);
  if (rc) return rc;
  if (k.type < 0 || k.type > 2) return fail(TBS_EINVAL, "kernel type %d unknown", k.type);
  if (k.type == TBS_K_GAUSSIAN && !std::isfinite(k.gamma)) return fail(TBS_EINVAL, "gamma must be finite");
  if (a->row_end > a->row_begin && !out) return fail(TBS_EINVAL, "out is NULL");
  if (a->row_end == a->row_begin || a->n == 0) return TBS_OK;
  cudaStream_t st = (cudaStream_t)a->stream;
  const int D = a->dim <= 3 ? 3 : 4;
  const int n_pad = pad_rows(a->n);
  float* soa = nullptr;
  uint32_t* bbox = nullptr;
  rc = load_points(a, D, n_pad, &soa, nullptr, 0, st, &bbox);
  if (!rc) {
    const float cexp = (float)(-(double)k.gamma * 1.4426950408889634);  // -gamma * log2(e)
    if (D == 3) rc = k.type == 0 ? matrix_launch<0, 3>(a, soa, n_pad, cexp, out, st)
                     : k.type == 1 ? matrix_launch<1, 3>(a, soa, n_pad, cexp, out, st)
                                   : matrix_launch<2, 3>(a, soa, n_pad, cexp, out, st);
    else rc = k.type == 0 ? matrix_launch<0, 4>(a, soa, n_pad, cexp, out, st)
              : k.type == 1 ? matrix_launch<1, 4>(a, soa, n_pad, cexp, out, st)
                            : matrix_launch<2, 4>(a, soa, n_pad, cexp, out, st);
  }
  release_soa(soa, st);
  return rc;
}

// ---- NEXT-3: high-dimensional Type-III on tcgen05 ---------------------------------------
using EncodeTiledFn = CUresult (*)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                   const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                                   CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

int encode_tiled_fn(EncodeTiledFn& fn) {
  static EncodeTiledFn cached = nullptr;
  if (!cached) {
    void* p = nullptr;
    cudaDriverEntryPointQueryResult q;
    TBS_CUDA(cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q));
    if (!p || q != cudaDriverEntryPointSuccess) return fail(TBS_ECUDA, "cuTensorMapEncodeTiled unavailable");
    cached = reinterpret_cast<EncodeTiledFn>(p);
  }
  fn = cached;
  return TBS_OK;
}

int hd_impl(const uint16_t* x, int64_t n, int d, int64_t rb, int64_t re, tbs_kernel k, float* out, cudaStream_t st,
            cudaEvent_t eb, cudaEvent_t ee) {
  if (n < 0 || n > (1 << 24)) return fail(TBS_EINVAL, "n out of range for the pair matrix");
  if (d < 1) return fail(TBS_EINVAL, "d must be >= 1");
  if (d > hd::kMaxD) return fail(TBS_EUNSUPPORTED, "d > %d not supported", hd::kMaxD);
  if (rb < 0 || re < rb || re > n) return fail(TBS_EINVAL, "row range outside [0, n]");
  if (k.type < 0 || k.type > 2) return fail(TBS_EINVAL, "kernel type %d unknown", k.type);
  if (k.type == TBS_K_GAUSSIAN && !std::isfinite(k.gamma)) return fail(TBS_EINVAL, "gamma must be finite");
  if (re > rb && (!x || !out)) return fail(TBS_EINVAL, "NULL features or output");
  if (re == rb) return TBS_OK;
  Device dev;
  int rc = current_device(dev);
  if (rc) return rc;
  // The CTA-pair kernel (256 x 256 tiles, half the L2 operand traffic per output, double-
  // buffered epilogue staging; tbs_hd2.cuh) is measured faster than the one-CTA 128 x 128
  // kernel (tbs_hd.cuh) at every d tried (64K points, d = 64: 3.10 vs 3.15 ms; d = 512:
  // 4.60 vs 6.26 ms); TBS_HD_1SM=1 selects the one-CTA kernel (A/B runs).
  static const bool one_sm = [] { const char* e = getenv("TBS_HD_1SM"); return e && atoi(e) != 0; }();
  const int dp = (d + hd::kKBlock - 1) / hd::kKBlock * hd::kKBlock;
  const int tile = one_sm ? hd::kTile : hd2::kPair;
  const int64_t n_pad = (n + tile - 1) / tile * tile;
  unsigned char* scratch = nullptr;
  const size_t xbytes = (size_t)n_pad * dp * 2;
  TBS_CUDA(cudaMallocAsync((void**)&scratch, xbytes + (size_t)n_pad * 4, st));
  uint16_t* xp = reinterpret_cast<uint16_t*>(scratch);
  float* norms = reinterpret_cast<float*>(scratch + xbytes);
  {
    const int threads = 256;
    const long long blocks = std::min<long long>((n_pad * 32 + threads - 1) / threads, (long long)dev.sms * 16);
    hd::hd_prep<<<(unsigned)blocks, threads, 0, st>>>(x, (int)n, d, (int)n_pad, dp, xp, norms);
    rc = cudaGetLastError() == cudaSuccess ? TBS_OK : fail(TBS_ECUDA, "hd_prep launch failed");
    g_launches.fetch_add(1);
  }
  EncodeTiledFn enc = nullptr;
  if (!rc) rc = encode_tiled_fn(enc);
  CUtensorMap tmap, tmap_out;
  const int use_tma_store = (n % 4) == 0;
  if (!rc) {
    const cuuint64_t dims[2] = {(cuuint64_t)dp, (cuuint64_t)n_pad};
    const cuuint64_t strides[1] = {(cuuint64_t)dp * 2};
    const cuuint32_t box[2] = {(cuuint32_t)hd::kKBlock, (cuuint32_t)hd::kTile};
    const cuuint32_t estr[2] = {1, 1};
    const CUresult cr = enc(&tmap, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, xp, dims, strides, box, estr,
                            CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
                            CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (cr != CUDA_SUCCESS) rc = fail(TBS_ECUDA, "cuTensorMapEncodeTiled failed (%d)", (int)cr);
  }
  if (!rc) {
    // output rows [rb, re) x n fp32; TMA boxes of 128 rows x 32 columns, 128-byte swizzle
    const cuuint64_t dims[2] = {(cuuint64_t)n, (cuuint64_t)(re - rb)};
    const cuuint64_t strides[1] = {(cuuint64_t)n * 4};
    const cuuint32_t box[2] = {(cuuint32_t)hd::kBoxCols, (cuuint32_t)hd::kTile};
    const cuuint32_t estr[2] = {1, 1};
    if (use_tma_store) {
      const CUresult cr = enc(&tmap_out, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, out, dims, strides, box, estr,
                              CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
                              CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
      if (cr != CUDA_SUCCESS) rc = fail(TBS_ECUDA, "cuTensorMapEncodeTiled (output) failed (%d)", (int)cr);
    } else {
      memset(&tmap_out, 0, sizeof(tmap_out));
    }
  }
  if (!rc) {
    const int I0 = (int)(rb / tile), I1 = (int)((re + tile - 1) / tile);
    const int tiles_i = I1 - I0, tiles_j = (int)(n_pad / tile);
    const long long ntiles = (long long)tiles_i * tiles_j;
    const int grid = one_sm ? (int)std::min<long long>(ntiles, dev.sms)
                            : 2 * (int)std::min<long long>(ntiles, dev.sms / 2);   // CTA pairs
    const float cexp = (float)(-(double)k.gamma * 1.4426950408889634);
    const int kblocks = dp / hd::kKBlock;
    // CTA-pair kernel shape (operand ring depth, epilogue staging buffers): small d (<= 2
    // k-blocks per tile, output-bound) vs large d.
    const bool small_d = kblocks <= 2;
    using SmemS = hd2::Smem<TBS_HD2_RING_S, TBS_HD2_NSTG_S>;
    using SmemL = hd2::Smem<TBS_HD2_RING_L, TBS_HD2_NSTG_L>;
    const int smem = (one_sm ? hd::Smem::BYTES : small_d ? SmemS::BYTES : SmemL::BYTES) + 1024;
    // CTA-pair tile raster: bands of `band` tile rows walked column by column, tiles dealt
    // round-robin over clusters (0: contiguous row-major range per cluster). TBS_HD_BAND overrides.
    static const int band_env = [] { const char* e = getenv("TBS_HD_BAND"); return e ? atoi(e) : -1; }();
    // Default: contiguous ranges for d <= 128 (output-bound; banding measured 3.19 vs 3.08 ms
    // at 64K x 64), else bands whose A rows hold ~8 MiB of features (64K x 512: band 32;
    // measured 8: 4.56, 16: 4.45, 32: 4.12, 64: 4.11, 128: 4.57, 256: 4.90 ms).
    const int band = band_env >= 0 ? band_env
                     : kblocks <= 2 ? 0
                                    : (int)std::max<long long>(1, (8ll << 20) / ((long long)hd2::kPair * dp * 2));
    auto launch = [&](auto kern) -> int {
      TBS_CUDA(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
      if (eb) TBS_CUDA(cudaEventRecord(eb, st));
      if constexpr (std::is_same<decltype(kern), decltype(&hd2::hd_pair_kernel<0, 4, 2>)>::value)
        kern<<<grid, hd2::kThreads, smem, st>>>(tmap, tmap_out, use_tma_store, norms, (int)n, kblocks, I0, tiles_i,
                                                tiles_j, (int)rb, (int)re, cexp, out, band);
      else
        kern<<<grid, hd::kThreads, smem, st>>>(tmap, tmap_out, use_tma_store, norms, (int)n, kblocks, I0, tiles_i,
                                               tiles_j, (int)rb, (int)re, cexp, out);
      TBS_CUDA(cudaGetLastError());
      g_launches.fetch_add(1);
      if (ee) TBS_CUDA(cudaEventRecord(ee, st));
      return TBS_OK;
    };
    if (one_sm)
      rc = k.type == 0 ? launch(hd::hd_pairmatrix_kernel<0>)
           : k.type == 1 ? launch(hd::hd_pairmatrix_kernel<1>)
                         : launch(hd::hd_pairmatrix_kernel<2>);
    else if (small_d)
      rc = k.type == 0 ? launch(hd2::hd_pair_kernel<0, TBS_HD2_RING_S, TBS_HD2_NSTG_S>)
           : k.type == 1 ? launch(hd2::hd_pair_kernel<1, TBS_HD2_RING_S, TBS_HD2_NSTG_S>)
                         : launch(hd2::hd_pair_kernel<2, TBS_HD2_RING_S, TBS_HD2_NSTG_S>);
    else
      rc = k.type == 0 ? launch(hd2::hd_pair_kernel<0, TBS_HD2_RING_L, TBS_HD2_NSTG_L>)
           : k.type == 1 ? launch(hd2::hd_pair_kernel<1, TBS_HD2_RING_L, TBS_HD2_NSTG_L>)
                         : launch(hd2::hd_pair_kernel<2, TBS_HD2_RING_L, TBS_HD2_NSTG_L>);
  }
  cudaFreeAsync(scratch, st);
  return rc;
}

// ---- NEXT-2: all-point kNN ---------------------------------------------------------------
#ifndef TBS_KNN8_KA
#define TBS_KNN8_KA 4   // anchors per thread for k <= 8 (A/B knob)
#endif
template <int K, int KA, int D>
int knn_launch(const Device& dev, const tbs_args* a, const float* soa, int n_pad, int k, int32_t* idx, float* dist,
               cudaStream_t st) {
  constexpr int TA = knn::kThreads * KA;
  auto kern = knn::knn_kernel<K, KA, D>;
  static thread_local int occ_dev = -1, occ = 0;
  if (occ_dev != dev.id) {
    TBS_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kern, knn::kThreads, 0));
    occ_dev = dev.id;
  }
  const int n = (int)a->n, rb = (int)a->row_begin, re = (int)a->row_end, rows = re - rb;
  const int I0 = rb / TA, tiles = (re + TA - 1) / TA - I0;
  const int n_chunks = (n + knn::kTP - 1) / knn::kTP;
  // partner segments so the grid is >= ~8 waves (wave-quantisation loss <= 1/8)
  const long long slots = (long long)dev.sms * std::max(occ, 1);
  int S = (int)std::min<long long>(std::max<long long>(1, (8 * slots + tiles - 1) / tiles), n_chunks);
  const int seg = (n_chunks + S - 1) / S;
  S = (n_chunks + seg - 1) / seg;
  float* ps = nullptr;
  int* pj = nullptr;
  if (S > 1) {
    TBS_CUDA(cudaMallocAsync((void**)&ps, (size_t)S * rows * K * 8, st));
    pj = reinterpret_cast<int*>(ps + (size_t)S * rows * K);
  }
  cudaEvent_t eb = (cudaEvent_t)a->ev_begin, ee = (cudaEvent_t)a->ev_end;
  int rc = TBS_OK;
  if (eb) TBS_CUDA(cudaEventRecord(eb, st));
  kern<<<dim3((unsigned)tiles, (unsigned)S), knn::kThreads, 0, st>>>(soa, n, n_pad, rb, re, I0, seg, n_chunks, k, ps, pj,
                                                                     idx, dist);
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) rc = fail(TBS_ECUDA, "knn_kernel: %s", cudaGetErrorString(e));
  g_launches.fetch_add(1);
  if (!rc && S > 1) {
    knn::knn_merge<K><<<(unsigned)((rows + 127) / 128), 128, 0, st>>>(ps, pj, rows, S, k, idx, dist);
    e = cudaGetLastError();
    if (e != cudaSuccess) rc = fail(TBS_ECUDA, "knn_merge: %s", cudaGetErrorString(e));
    g_launches.fetch_add(1);
  }
  if (!rc && ee) TBS_CUDA(cudaEventRecord(ee, st));
  if (ps) cudaFreeAsync(ps, st);
  return rc;
}

int knn_impl(const tbs_args* a, int k, int32_t* idx, float* dist) {
  int rc = validate_common(a);
  if (rc) return rc;
  if (k < 1 || k > TBS_KNN_MAX_K) return fail(TBS_EINVAL, "k = %d outside [1, %d]", k, TBS_KNN_MAX_K);
  if (a->row_end > a->row_begin && (!idx || !dist)) return fail(TBS_EINVAL, "idx or dist is NULL");
  if (a->row_end == a->row_begin) return TBS_OK;
  Device dev;
  if ((rc = current_device(dev))) return rc;
  cudaStream_t st = (cudaStream_t)a->stream;
  const int D = a->dim <= 3 ? 3 : 4;
  const int n_pad = pad_rows(a->n);
  float* soa = nullptr;
  uint32_t* bbox = nullptr;
  rc = load_points(a, D, n_pad, &soa, nullptr, 0, st, &bbox, INFINITY);
  if (!rc) {
    if (D == 3) rc = k <= 4 ? knn_launch<4, 4, 3>(dev, a, soa, n_pad, k, idx, dist, st)
                     : k <= 8 ? knn_launch<8, TBS_KNN8_KA, 3>(dev, a, soa, n_pad, k, idx, dist, st)
                     : k <= 16 ? knn_launch<16, 2, 3>(dev, a, soa, n_pad, k, idx, dist, st)
                               : knn_launch<32, 2, 3>(dev, a, soa, n_pad, k, idx, dist, st);
    else rc = k <= 4 ? knn_launch<4, 4, 4>(dev, a, soa, n_pad, k, idx, dist, st)
              : k <= 8 ? knn_launch<8, TBS_KNN8_KA, 4>(dev, a, soa, n_pad, k, idx, dist, st)
              : k <= 16 ? knn_launch<16, 2, 4>(dev, a, soa, n_pad, k, idx, dist, st)
                        : knn_launch<32, 2, 4>(dev, a, soa, n_pad, k, idx, dist, st);
  }
  release_soa(soa, st);
  return rc;
}

// ---- host-or-device simple entry points ------------------------------------------
// Where a pointer lives: 0 pageable host, 1 page-locked (pinned) host, 2 device / managed.
int pointer_kind(const void* p, int& kind) {
  kind = 0;
  if (!p) return TBS_OK;
  cudaPointerAttributes at;
  cudaError_t e = cudaPointerGetAttributes(&at, p);
  if (e != cudaSuccess) {
    cudaGetLastError();
    return TBS_OK;  // unregistered host memory
  }
  kind = (at.type == cudaMemoryTypeDevice || at.type == cudaMemoryTypeManaged) ? 2
         : at.type == cudaMemoryTypeHost ? 1 : 0;
  return TBS_OK;
}
int is_device_ptr(const void* p, bool& dev) {
  int k = 0;
  const int rc = pointer_kind(p, k);
  dev = k == 2;
  return rc;
}

// Per-thread page-locked staging for pageable host buffers of the simple entry points (a copy
// from pageable memory is staged by the driver synchronously, chunk by chunk; a memcpy into a
// cached pinned buffer plus one DMA is faster for the small calls this path serves).
struct Staging {
  void* p = nullptr;
  size_t bytes = 0;
  ~Staging() { if (p) cudaFreeHost(p); }
};
int staging(size_t bytes, void** out) {
  static thread_local Staging s;
  if (s.bytes < bytes) {
    if (s.p) cudaFreeHost(s.p);
    s.p = nullptr;
    s.bytes = 0;
    const size_t want = std::max<size_t>(bytes, 1 << 20);
    if (cudaHostAlloc(&s.p, want, cudaHostAllocPortable | cudaHostAllocMapped) != cudaSuccess) {
      cudaGetLastError();
      return fail(TBS_ENOMEM, "cudaHostAlloc(%zu) for host staging failed", want);
    }
    s.bytes = want;
  }
  *out = s.p;
  return TBS_OK;
}

// TBS_HOST_TRACE (diagnostics): per-phase host time of the small host-buffer path, averaged over
// the calls and printed to stderr at exit.
struct HostTrace {
  static constexpr int kPhases = 8;
  double ns[kPhases] = {0};
  long long calls = 0;
  std::chrono::steady_clock::time_point t;
  bool on = getenv("TBS_HOST_TRACE") != nullptr;
  void start() { if (on) t = std::chrono::steady_clock::now(); }
  void mark(int k) {
    if (!on) return;
    const auto now = std::chrono::steady_clock::now();
    ns[k] += std::chrono::duration<double, std::nano>(now - t).count();
    t = now;
  }
  ~HostTrace() {
    if (!on || !calls) return;
    static const char* names[kPhases] = {"pointer_kind", "staging+memcpy", "host_dev_ptr", "malloc_async", "copy_kernel",
                                         "op_call", "free_async", "poll"};
    fprintf(stderr, "[tbs host trace] %lld calls, us per call:", calls);
    for (int k = 0; k < kPhases; ++k) fprintf(stderr, " %s %.2f", names[k], ns[k] / calls * 1e-3);
    fprintf(stderr, "\n");
  }
};
HostTrace& host_trace() {
  static HostTrace h;
  return h;
}

// Per-thread device scratch of the small host-buffer path: [output | ticket], kept ZERO between
// calls (zeroed once when allocated; afterwards the fused kernel's last CTA re-zeroes what the
// call used, or the call itself on its fallback and error paths), so a call needs no allocation,
// memset or copy kernel before its one launch.
struct SmallScratch {
  int dev = -1;
  unsigned char* p = nullptr;
  size_t bytes = 0;
};
int small_scratch(size_t bytes, unsigned char** out) {
  constexpr int kDevs = 16;
  static thread_local SmallScratch per_dev[kDevs];   // one buffer per device and thread
  int d = 0;
  TBS_CUDA(cudaGetDevice(&d));
  if (d < 0 || d >= kDevs) return fail(TBS_EUNSUPPORTED, "small host path: device %d >= %d", d, kDevs);
  SmallScratch& s = per_dev[d];
  if (s.bytes < bytes) {
    const size_t want = std::max<size_t>(bytes, 65536 + 64 + 16384 * 16);   // output region + the largest points
    unsigned char* p = nullptr;
    TBS_CUDA(cudaMalloc((void**)&p, want));
    TBS_CUDA(cudaMemset(p, 0, want));
    if (s.p) cudaFree(s.p);   // (synchronous; the previous call on this thread has completed)
    s = SmallScratch{d, p, want};
  }
  *out = s.p;
  return TBS_OK;
}
// The points are pulled into device memory by a copy kernel first. TBS_SMALL_DIRECT=1 (A/B):
// the fused kernel reads them from the mapped host buffer instead — measured slower (46 vs
// 32.8 us per N = 4096 call: its 144 CTAs re-read the same lines over the host link).
bool small_copy_in() {
  static const bool v = [] { const char* e = getenv("TBS_SMALL_DIRECT"); return !(e && atoi(e) != 0); }();
  return v;
}

// Run `fn(args_with_device_ptrs, dev_out)` for host or device buffers, synchronously.
template <class Fn>
int run_simple(const float* points, int64_t n, int dim, void* outp, size_t out_bytes, Fn fn,
               bool small_op = false) {
  if (n < 0 || n > TBS_MAX_N) return fail(TBS_EINVAL, "n out of range");
  if (dim < 1 || dim > 4) return fail(TBS_EINVAL, "dim out of range");
  if (!outp) return fail(TBS_EINVAL, "output is NULL");
  if (n >= 2 && !points) return fail(TBS_EINVAL, "points is NULL");
  int pk = 0, ok = 0;
  HostTrace& tr = host_trace();
  tr.start();
  int rc = pointer_kind(points, pk);
  if (!rc) rc = pointer_kind(outp, ok);
  if (rc) return rc;
  tr.mark(0);
  if (points && (pk == 2) != (ok == 2)) return fail(TBS_EINVAL, "points and output must both be host or both device pointers");
  cudaStream_t st = cudaStreamPerThread;
  tbs_args a{};
  a.n = n;
  a.dim = dim;
  a.row_begin = 0;
  a.row_end = n;
  a.stream = st;
  if (ok == 2) {
    a.points = points;
    rc = fn(&a, outp);
    if (!rc) TBS_CUDA(cudaStreamSynchronize(st));
    return rc;
  }
  const size_t pbytes = (size_t)n * dim * sizeof(float);
  if (small_op && n >= 2 && n <= kSmallLoad && out_bytes <= 65536 && out_bytes % 8 == 0) {
    // Small problem: the copy engines' two transfers cost more than the ~10 us kernel. The
    // points are pulled from pinned host memory (the caller's, or the staging area) by a copy
    // kernel and the result is pushed back the same way: every step is a kernel on one stream.
    // staging: [points (pageable input) | output (pageable output) | completion flag]
    const size_t pin_in = pk == 1 ? 0 : (pbytes + 255) / 256 * 256;
    const size_t pin_out = ok == 1 ? 0 : (out_bytes + 255) / 256 * 256;
    unsigned char* stage = nullptr;
    {
      void* sp = nullptr;
      if ((rc = staging(pin_in + pin_out + 64, &sp))) return rc;
      stage = static_cast<unsigned char*>(sp);
    }
    volatile unsigned int* flag = reinterpret_cast<volatile unsigned int*>(stage + pin_in + pin_out);
    void* dflag = nullptr;
    const void* src = points;
    if (pin_in) {
      memcpy(stage, points, pbytes);
      src = stage;
    }
    void* dst = pin_out ? static_cast<void*>(stage + pin_in) : outp;
    void *dsrc = nullptr, *ddst = nullptr;
    tr.mark(1);
    if (cudaHostGetDevicePointer(&dsrc, const_cast<void*>(src), 0) == cudaSuccess &&
        cudaHostGetDevicePointer(&ddst, dst, 0) == cudaSuccess &&
        cudaHostGetDevicePointer(&dflag, const_cast<unsigned int*>(flag), 0) == cudaSuccess) {
      tr.mark(2);
      // [output + ticket region (fixed, 64 KB + 64 B: zero on entry) | points (copy-in variant)]:
      // the output and the ticket sit at the same place whatever the call's sizes, so the points
      // of one call never land where a later call expects zeros
      constexpr size_t kOutRegion = 65536 + 64;
      const size_t dp_bytes = small_copy_in() ? (pbytes + 255) / 256 * 256 : 0;
      unsigned char* dscr = nullptr;
      if ((rc = small_scratch(kOutRegion + dp_bytes, &dscr))) return rc;
      tr.mark(3);
      const int in_words = (int)(pbytes / 4), out_words = (int)(out_bytes / 4);
      unsigned char* dout = dscr;
      unsigned char* dbuf = dscr + kOutRegion;
      if (dp_bytes) {
        copy_in_zero<<<(in_words + 1023) / 1024 < 8 ? (in_words + 1023) / 1024 : 8, 1024, 0, st>>>(
            reinterpret_cast<uint32_t*>(dbuf), static_cast<const uint32_t*>(dsrc), in_words,
            reinterpret_cast<uint32_t*>(dout), 0);
        g_launches.fetch_add(1);
      }
      tr.mark(4);
      // the fused kernel reads the points straight from the mapped page-locked host buffer
      a.points = dp_bytes ? reinterpret_cast<const float*>(dbuf) : static_cast<const float*>(dsrc);
      SmallWriteBack& sw = small_wb();
      sw.wb.dst = static_cast<unsigned long long*>(ddst);
      sw.wb.src = reinterpret_cast<unsigned long long*>(dout);
      sw.wb.rezero = 1;
      sw.wb.ticket = reinterpret_cast<unsigned int*>(dout + out_bytes);
      sw.wb.words = (int)(out_bytes / 8);
      static thread_local unsigned int seq = 0;
      seq = seq + 1 == 0 ? 1 : seq + 1;
      *flag = 0u;
      sw.wb.flag = static_cast<unsigned int*>(dflag);
      sw.wb.seq = seq;
      sw.active = true;
      sw.taken = false;
      rc = fn(&a, dout);
      tr.mark(5);
      const bool taken = sw.taken;
      sw = SmallWriteBack{};
      if (!rc && !taken) {
        copy_words<<<1, 256, 0, st>>>(static_cast<uint32_t*>(ddst), reinterpret_cast<const uint32_t*>(dout), out_words);
        g_launches.fetch_add(1);
      }
      if (rc || !taken) cudaMemsetAsync(dout, 0, out_bytes + 8, st);   // restore the zero scratch
      tr.mark(6);
      bool done = false;
      if (!rc && taken) {
        // the kernel's last CTA signals completion through the mapped flag: poll it (a stream
        // synchronisation costs a host wake-up); give up to the synchronisation after ~50 ms
        const auto t0 = std::chrono::steady_clock::now();
        while (!(done = *flag == seq)) {
          if (std::chrono::steady_clock::now() - t0 > std::chrono::milliseconds(50)) break;
        }
      }
      if (!done) {
        const cudaError_t e = cudaStreamSynchronize(st);
        if (!rc && e != cudaSuccess) rc = fail(TBS_ECUDA, "sync: %s", cudaGetErrorString(e));
      }
      if (!rc && pin_out) memcpy(outp, dst, out_bytes);
      tr.mark(7);
      if (tr.on) tr.calls++;
      return rc;
    }
    cudaGetLastError();   // not mapped: the copy-engine path below
  }
  // pageable buffers go through the pinned staging area: [points | output]
  size_t pin_in = pk == 1 ? 0 : (pbytes + 255) / 256 * 256;
  size_t pin_out = ok == 1 ? 0 : out_bytes;
  if (pin_in + pin_out > ((size_t)64 << 20)) pin_in = pin_out = 0;   // large: the driver's own staging
  unsigned char* stage = nullptr;
  if (pin_in + pin_out) {
    void* sp = nullptr;
    if ((rc = staging(pin_in + pin_out, &sp))) return rc;
    stage = static_cast<unsigned char*>(sp);
  }
  const void* src = points;
  if (pin_in && pbytes) {
    memcpy(stage, points, pbytes);
    src = stage;
  }
  void* dst_host = pin_out ? static_cast<void*>(stage + pin_in) : outp;
  // one device allocation: [points | output]
  const size_t dp_bytes = (pbytes + 255) / 256 * 256;
  unsigned char* dbuf = nullptr;
  cudaError_t e = cudaMallocAsync((void**)&dbuf, dp_bytes + std::max<size_t>(out_bytes, 4), st);
  if (e != cudaSuccess) return fail(TBS_ENOMEM, "cudaMallocAsync(%zu): %s", dp_bytes + out_bytes, cudaGetErrorString(e));
  float* dp = reinterpret_cast<float*>(dbuf);
  void* dout = dbuf + dp_bytes;
  if (pbytes) e = cudaMemcpyAsync(dp, src, pbytes, cudaMemcpyHostToDevice, st);
  a.points = dp;
  rc = e != cudaSuccess ? fail(TBS_ECUDA, "H2D copy: %s", cudaGetErrorString(e)) : fn(&a, dout);
  if (!rc) {
    e = cudaMemcpyAsync(dst_host, dout, out_bytes, cudaMemcpyDeviceToHost, st);
    if (e != cudaSuccess) rc = fail(TBS_ECUDA, "D2H copy: %s", cudaGetErrorString(e));
  }
  cudaFreeAsync(dbuf, st);
  e = cudaStreamSynchronize(st);
  if (!rc && e != cudaSuccess) rc = fail(TBS_ECUDA, "sync: %s", cudaGetErrorString(e));
  if (!rc && pin_out) memcpy(outp, dst_host, out_bytes);
  return rc;
}

}  // namespace

extern "C" {

int tbs_sdh_ex(const tbs_args* args, float bucket_width, int nbuckets, uint64_t* hist) {
  g_err.clear();
  return sdh_impl(args, bucket_width, nbuckets, hist);
}

int tbs_pcf_ex(const tbs_args* args, float radius, uint64_t* count) {
  g_err.clear();
  return pcf_impl(args, radius, count);
}

int tbs_pairmatrix_ex(const tbs_args* args, tbs_kernel kernel, float* out) {
  g_err.clear();
  return pairmatrix_impl(args, kernel, out);
}

int tbs_sdh(const float* points, int64_t n, int dim, float bucket_width, int nbuckets, uint64_t* hist) {
  g_err.clear();
  if (nbuckets < 1 || nbuckets > TBS_MAX_BUCKETS) return fail(TBS_EINVAL, "nbuckets out of range");
  return run_simple(points, n, dim, hist, (size_t)nbuckets * 8, [&](tbs_args* a, void* out) {
    return sdh_impl(a, bucket_width, nbuckets, (uint64_t*)out);
  }, true);
}

int tbs_pcf(const float* points, int64_t n, float radius, uint64_t* count) {
  g_err.clear();
  return run_simple(points, n, 3, count, 8, [&](tbs_args* a, void* out) { return pcf_impl(a, radius, (uint64_t*)out); },
                    true);
}

int tbs_pairmatrix(const float* points, int64_t n, tbs_kernel kernel, float* out) {
  g_err.clear();
  if (n < 0 || n > TBS_MAX_N) return fail(TBS_EINVAL, "n out of range");
  return run_simple(points, n, 3, out, (size_t)n * (size_t)n * sizeof(float) + (n == 0 ? 4 : 0),
                    [&](tbs_args* a, void* o) { return pairmatrix_impl(a, kernel, (float*)o); });
}

int tbs_kde_ex(const tbs_args* args, float gamma, double* sum) {
  g_err.clear();
  return kde_impl(args, gamma, sum);
}

int tbs_kde(const float* points, int64_t n, float gamma, double* sum) {
  g_err.clear();
  return run_simple(points, n, 3, sum, 8, [&](tbs_args* a, void* out) { return kde_impl(a, gamma, (double*)out); }, true);
}

int tbs_rdf_ex(const tbs_args* args, float bucket_width, int nbuckets, double volume, double* g) {
  g_err.clear();
  return rdf_impl(args, bucket_width, nbuckets, volume, g);
}

int tbs_rdf_hist_ex(const uint64_t* hist, int nbuckets, int dim, float bucket_width, double pairs, double volume,
                    double* g, void* stream) {
  g_err.clear();
  int rc = rdf_args_ok(nbuckets, dim, bucket_width, volume, g);
  if (rc) return rc;
  if (!hist) return fail(TBS_EINVAL, "hist is NULL");
  if (!(pairs >= 0.0) || !std::isfinite(pairs)) return fail(TBS_EINVAL, "pairs must be finite and >= 0");
  return rdf_normalize(hist, nbuckets, dim, bucket_width, pairs, volume, g, (cudaStream_t)stream);
}

int tbs_rdf(const float* points, int64_t n, int dim, float bucket_width, int nbuckets, double volume, double* g) {
  g_err.clear();
  if (nbuckets < 1 || nbuckets >= TBS_MAX_BUCKETS) return fail(TBS_EINVAL, "nbuckets out of range");
  return run_simple(points, n, dim, g, (size_t)nbuckets * 8, [&](tbs_args* a, void* out) {
    return rdf_impl(a, bucket_width, nbuckets, volume, (double*)out);
  });
}

int tbs_pairmatrix_hd_ex(const uint16_t* features, int64_t n, int d, int64_t row_begin, int64_t row_end,
                         tbs_kernel kernel, float* out, void* stream, void* ev_begin, void* ev_end) {
  g_err.clear();
  return hd_impl(features, n, d, row_begin, row_end, kernel, out, (cudaStream_t)stream, (cudaEvent_t)ev_begin,
                 (cudaEvent_t)ev_end);
}

int tbs_pairmatrix_hd(const uint16_t* features, int64_t n, int d, tbs_kernel kernel, float* out) {
  g_err.clear();
  if (n < 0 || d < 1 || !out || (n > 0 && !features)) return fail(TBS_EINVAL, "tbs_pairmatrix_hd: bad arguments");
  bool fdev = false, odev = false;
  is_device_ptr(features, fdev);
  is_device_ptr(out, odev);
  if (n > 0 && fdev != odev) return fail(TBS_EINVAL, "features and out must both be host or both device pointers");
  cudaStream_t st = cudaStreamPerThread;
  if (odev) {
    int rc = hd_impl(features, n, d, 0, n, kernel, out, st, nullptr, nullptr);
    if (!rc) TBS_CUDA(cudaStreamSynchronize(st));
    return rc;
  }
  uint16_t* df = nullptr;
  float* dout = nullptr;
  const size_t fb = (size_t)n * d * 2, ob = (size_t)n * n * 4;
  if (fb) TBS_CUDA(cudaMallocAsync((void**)&df, fb, st));
  cudaError_t e = cudaMallocAsync((void**)&dout, ob ? ob : 4, st);
  if (e != cudaSuccess) {
    if (df) cudaFreeAsync(df, st);
    return fail(TBS_ENOMEM, "cudaMallocAsync(%zu): %s", ob, cudaGetErrorString(e));
  }
  if (fb) e = cudaMemcpyAsync(df, features, fb, cudaMemcpyHostToDevice, st);
  int rc = e != cudaSuccess ? fail(TBS_ECUDA, "H2D: %s", cudaGetErrorString(e))
                            : hd_impl(df, n, d, 0, n, kernel, dout, st, nullptr, nullptr);
  if (!rc && ob) {
    e = cudaMemcpyAsync(out, dout, ob, cudaMemcpyDeviceToHost, st);
    if (e != cudaSuccess) rc = fail(TBS_ECUDA, "D2H: %s", cudaGetErrorString(e));
  }
  if (df) cudaFreeAsync(df, st);
  cudaFreeAsync(dout, st);
  e = cudaStreamSynchronize(st);
  if (!rc && e != cudaSuccess) rc = fail(TBS_ECUDA, "sync: %s", cudaGetErrorString(e));
  return rc;
}

int tbs_knn_ex(const tbs_args* args, int k, int32_t* idx, float* dist) {
  g_err.clear();
  return knn_impl(args, k, idx, dist);
}

int tbs_knn(const float* points, int64_t n, int dim, int k, int32_t* idx, float* dist) {
  g_err.clear();
  if (n < 0 || n > TBS_MAX_N || k < 1 || k > TBS_KNN_MAX_K || !idx || !dist)
    return fail(TBS_EINVAL, "tbs_knn: bad arguments");
  const size_t half = (size_t)n * (size_t)k * 4;
  bool ddev = false;
  is_device_ptr(dist, ddev);
  if (ddev) {
    bool idev = false;
    is_device_ptr(idx, idev);
    if (!idev) return fail(TBS_EINVAL, "idx and dist must both be host or both device pointers");
    return run_simple(points, n, dim, dist, half, [&](tbs_args* a, void*) { return knn_impl(a, k, idx, dist); });
  }
  // host buffers: one device allocation holds [idx | dist]; copy both halves back
  std::vector<unsigned char> both(2 * half + 4);
  int rc = run_simple(points, n, dim, both.data(), 2 * half + 4, [&](tbs_args* a, void* o) {
    return knn_impl(a, k, reinterpret_cast<int32_t*>(o),
                    reinterpret_cast<float*>(reinterpret_cast<unsigned char*>(o) + half));
  });
  if (!rc && half) {
    std::memcpy(idx, both.data(), half);
    std::memcpy(dist, both.data() + half, half);
  }
  return rc;
}

int tbs_rank_rows(int64_t n, int world, int rank, int64_t* row_begin, int64_t* row_end) {
  g_err.clear();
  if (n < 0 || world < 1 || rank < 0 || rank >= world || !row_begin || !row_end)
    return fail(TBS_EINVAL, "tbs_rank_rows: bad arguments");
  // S(R) = sum_{i<R} (n-1-i) = R(2n-R-1)/2 pairs have anchors below row R. Boundary r
  // solves S(R) = r * P / world, P = n(n-1)/2; take the integer R whose S is nearest.
  auto boundary = [&](int r) -> int64_t {
    if (r <= 0) return 0;
    if (r >= world) return n;
    const __int128 P = (__int128)n * (n - 1) / 2;
    const __int128 target = P * r / world;
    const double b = 2.0 * (double)n - 1.0;
    double R = 0.5 * (b - std::sqrt(std::max(0.0, b * b - 8.0 * (double)target)));
    int64_t Ri = std::min<int64_t>(std::max<int64_t>((int64_t)R, 0), n);
    auto S = [&](int64_t x) { return (__int128)x * (2 * n - x - 1) / 2; };
    while (Ri > 0 && S(Ri) > target) --Ri;
    while (Ri < n && S(Ri + 1) <= target) ++Ri;
    if (Ri < n && (S(Ri + 1) - target) < (target - S(Ri))) ++Ri;
    return Ri;
  };
  *row_begin = boundary(rank);
  *row_end = boundary(rank + 1);
  return TBS_OK;
}

int tbs_peer_alloc(uint64_t bytes, void** dev_ptr, void* handle) {
  if (!dev_ptr || !handle || bytes == 0) return fail(TBS_EINVAL, "tbs_peer_alloc: bad arguments");
  void* p = nullptr;
  cudaError_t e = cudaMalloc(&p, (size_t)bytes);
  if (e == cudaErrorMemoryAllocation) return fail(TBS_ENOMEM, "tbs_peer_alloc: %s", cudaGetErrorString(e));
  TBS_CUDA(e);
  TBS_CUDA(cudaMemset(p, 0, (size_t)bytes));
  cudaIpcMemHandle_t h;
  TBS_CUDA(cudaIpcGetMemHandle(&h, p));
  static_assert(sizeof(h) == 64, "IPC handle size");
  memcpy(handle, &h, sizeof(h));
  *dev_ptr = p;
  return TBS_OK;
}

int tbs_peer_open(const void* handle, void** dev_ptr) {
  if (!dev_ptr || !handle) return fail(TBS_EINVAL, "tbs_peer_open: bad arguments");
  cudaIpcMemHandle_t h;
  memcpy(&h, handle, sizeof(h));
  TBS_CUDA(cudaIpcOpenMemHandle(dev_ptr, h, cudaIpcMemLazyEnablePeerAccess));
  return TBS_OK;
}

int tbs_peer_close(void* dev_ptr) {
  TBS_CUDA(cudaIpcCloseMemHandle(dev_ptr));
  return TBS_OK;
}

int tbs_peer_free(void* dev_ptr) {
  TBS_CUDA(cudaFree(dev_ptr));
  return TBS_OK;
}

int tbs_peer_atomics_ok(const char* pci_bus_id, int* ok) {
  g_err.clear();
  if (!pci_bus_id || !ok) return fail(TBS_EINVAL, "tbs_peer_atomics_ok: bad arguments");
  *ok = 0;
  int self = 0, peer = -1;
  TBS_CUDA(cudaGetDevice(&self));
  if (cudaDeviceGetByPCIBusId(&peer, pci_bus_id) != cudaSuccess) {
    cudaGetLastError();
    return TBS_OK;   // not visible to this process: no peer access to query
  }
  if (peer == self) {
    *ok = 1;          // the same GPU (e.g. two processes on one device): device-local atomics
    return TBS_OK;
  }
  int access = 0, atomics = 0;
  TBS_CUDA(cudaDeviceCanAccessPeer(&access, self, peer));
  TBS_CUDA(cudaDeviceGetP2PAttribute(&atomics, cudaDevP2PAttrNativeAtomicSupported, self, peer));
  *ok = (access && atomics) ? 1 : 0;
  return TBS_OK;
}

const char* tbs_last_error(void) { return g_err.c_str(); }

void tbs_release(void) {
  int dev;
  if (cudaGetDevice(&dev) != cudaSuccess) return;
  cudaMemPool_t pool;
  if (cudaDeviceGetDefaultMemPool(&pool, dev) == cudaSuccess) {
    cudaDeviceSynchronize();
    cudaMemPoolTrimTo(pool, 0);
  }
}

uint64_t tbs_launch_count(void) { return g_launches.load(); }

int tbs_version(void) { return 200; }

}  // extern "C"
