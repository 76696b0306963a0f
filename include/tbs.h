/*
 * tbs.h — C ABI of the B200-native 2-body-statistics (2-BS) library, libtbs.so.
 *
 * The operations are the three output types of Pitaksirianan, Nouri & Tu,
 * "Efficient 2-Body Statistics Computation on GPUs" (ICPP 2016). Citations are to
 * /root/reference/PAPER.md lines (L<a>-<b>) with the section they fall in.
 *
 *   2-BS (§I): a statistic over all pairs of an N-point set computed from a
 *   pairwise "distance function". Every unordered pair {i, j}, i != j, contributes
 *   exactly once (Alg. 1 loops i = t+1..N, L290-296; Alg. 2).
 *   Distance = Euclidean (L600-602, L841-843).
 *
 *   tbs_sdh        Type-II output (§III-B, §IV-D): the spatial
 *                  distance histogram, hist[k] = #{i<j : min(floor(d_ij / w), nb-1) = k}.
 *   tbs_pcf        Type-I output (§III-B, §IV-B): the 2-point
 *                  correlation count, #{i<j : d_ij < r}.
 *   tbs_pairmatrix Type-III output (§III-B, §IV-C): the full pairwise
 *                  kernel matrix out[i][j] = K(p_i, p_j), diagonal included.
 *
 * Readings of points the paper leaves open are listed in DESIGN.md §Readings
 * (half-open buckets, clamping of d >= nb*w into the last bucket, d < r for 2PCF,
 * Gaussian kernel for Type-III).
 *
 * ---- Memory and ownership --------------------------------------------------------
 * points   AoS float32 [n][dim], row-major, read-only, caller-owned.
 * hist     uint64 [nbuckets], caller-allocated, OVERWRITTEN (not accumulated).
 * count    uint64 [1], caller-allocated, overwritten.
 * out      float32 [row_end - row_begin][n] row-major, caller-allocated, overwritten.
 * The simple entry points (tbs_sdh, tbs_pcf, tbs_pairmatrix) accept HOST or DEVICE
 * pointers (detected with cudaPointerGetAttributes; all arrays of one call must be
 * on the same side), run on a library stream and return after the result is in
 * place (synchronous). The _ex entry points take DEVICE pointers only, enqueue on
 * args->stream and return without synchronising: results are valid once that
 * stream has been synchronised. Scratch (the SoA coordinate copy, partial
 * histograms) is allocated stream-ordered from the device's default memory pool
 * and returned to it at the end of each call; tbs_release() trims the pool.
 *
 * ---- Errors ------------------------------------------------------------------------
 * Every function returns a tbs_status. Argument errors are detected synchronously,
 * return TBS_EINVAL and enqueue nothing: n < 0 or n > TBS_MAX_N; dim outside [1,4];
 * nbuckets < 1 or > TBS_MAX_BUCKETS; bucket_width <= 0 or non-finite; radius < 0 or
 * NaN; NULL array with n >= 2 (or a NULL output); a row range outside [0, n];
 * TBS_EXACT_LATTICE with a bucket width that is not m * 2^-j (m, j integers,
 * 1 <= m, (nbuckets + 1) * m < 2^31, 0 <= j <= 19). n < 2 (or an empty row range) is valid and yields
 * zero output. Allocation failure returns TBS_ENOMEM; a CUDA error returns
 * TBS_ECUDA. tbs_last_error() gives a thread-local message for the last non-OK
 * status. Non-finite coordinates are a caller contract violation (not checked on
 * the hot path; TBS_VALIDATE checks them). Under TBS_EXACT_LATTICE, coordinates must be
 * integer-valued with every squared pair distance < 2^24 (exact in fp32) and 4^j * s < 2^62
 * (TBS_VALIDATE checks the first two).
 */
#ifndef TBS_H_
#define TBS_H_

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
  TBS_OK = 0,
  TBS_EINVAL = 1,
  TBS_ENOMEM = 2,
  TBS_ECUDA = 3,
  TBS_EUNSUPPORTED = 4
} tbs_status;

/* Type-III pair functions. TBS_K_GAUSSIAN is exp(-gamma * ||x - y||^2) (reading Q10). */
typedef enum { TBS_K_GAUSSIAN = 0, TBS_K_DIST2 = 1, TBS_K_DIST = 2 } tbs_kernel_type;
typedef struct {
  int type;     /* tbs_kernel_type */
  float gamma;  /* TBS_K_GAUSSIAN only */
} tbs_kernel;

/* Flags for tbs_args.flags. */
#define TBS_EXACT_LATTICE 0x1u        /* SDH: exact integer squared-distance bucketing   */
#define TBS_HIST_FORCE_LANE 0x10u     /* SDH: 32 lane-private smem copies per CTA          */
#define TBS_HIST_FORCE_CTA 0x20u      /* SDH: one shared smem copy per CTA                 */
#define TBS_HIST_FORCE_GLOBAL 0x40u   /* SDH: partially privatised global u64 copies       */
#define TBS_FORCE_CLAMP 0x100u        /* SDH: never elide the nb-1 clamp (ablation/tests)   */
#define TBS_HIST_FORCE_PASSES 0x200u  /* SDH: bucket-range passes with one smem copy (tests)   */
/* SDH / 2PCF: fused multi-GPU combine (the paper's multi-GPU future work,
 * L1254-1256). Instead of writing hist / count, the call accumulates its (row-range) partial in
 * a local device buffer and adds that partial with system-scope atomics into EACH of
 * args->out_peers[0 .. n_out_peers) — inside the pair kernel itself (its last CTA to finish,
 * for single-launch output stages: smem-copy SDH, 2PCF) or, after multi-launch stages (bucket
 * passes, global partials, the small fused path), in one extra kernel — uint64 [out_peer_words] device buffers,
 * out_peer_words = nb (SDH) or 1 (2PCF): the local rank's own and the other ranks' mapped over
 * NVLink by CUDA IPC (tbs_peer_open; peers need native atomics, tbs_peer_atomics_ok). That is
 * out_peer_words x n_out_peers remote adds per rank. Nothing is zeroed: the caller zeroes
 * every rank's buffer before any rank's call starts, and after every rank's call has completed
 * each buffer holds the sum over all ranks' row ranges (the all-reduce, without a separate
 * collective). hist / count may be NULL. Other entry points return TBS_EUNSUPPORTED. */
#define TBS_OUT_PEERS 0x400u
/* Debug validation: the loader's pass over the points also records non-finite
 * and non-integer coordinates and the bounding box; with TBS_VALIDATE the call waits for it
 * (one stream synchronisation) and returns TBS_EINVAL, before any pair kernel runs, if a
 * coordinate is non-finite or, under TBS_EXACT_LATTICE, non-integer or spread so far that a
 * squared pair distance could reach 2^24 (sum over the coordinates of (max - min)^2 >= 2^24).
 * Not for the hot path: it costs a host round trip. SDH, 2PCF, kernel density, RDF. */
#define TBS_VALIDATE 0x800u

#define TBS_MAX_N ((int64_t)1 << 30)
#define TBS_MAX_BUCKETS (1 << 24)

/* ---- simple entry points (north-star signatures), host or device pointers -------- */

/* SDH over all pairs of points[n][dim]: hist[k] = #{i<j : min(floor(d/w), nb-1) = k}. */
int tbs_sdh(const float* points, int64_t n, int dim, float bucket_width, int nbuckets, uint64_t* hist);

/* 2PCF over all pairs of points[n][3]: *count = #{i<j : d < radius}. */
int tbs_pcf(const float* points, int64_t n, float radius, uint64_t* count);

/* Type-III over points[n][3]: out[i*n + j] = K(p_i, p_j) for all i, j in [0, n). */
int tbs_pairmatrix(const float* points, int64_t n, tbs_kernel kernel, float* out);

/* ---- extended entry points: device pointers, caller stream, row ranges ------------- */
typedef struct {
  const float* points;  /* device AoS float32 [n][dim]                                     */
  int64_t n;
  int dim;              /* 1..4                                                            */
  int64_t row_begin;    /* anchors i in [row_begin, row_end) pair with every j > i          */
  int64_t row_end;      /* (Type-III: rows i in [row_begin,row_end) against all j in [0,n)) */
  void* stream;         /* cudaStream_t; NULL = legacy default stream                      */
  uint32_t flags;       /* TBS_* flags above                                               */
  void* ev_begin;       /* optional cudaEvent_t recorded just before the pair kernel        */
  void* ev_end;         /* optional cudaEvent_t recorded just after it (profiling hook)     */
  void* const* out_peers; /* TBS_OUT_PEERS: device pointers of every rank's output buffer     */
  int n_out_peers;      /* 1 .. TBS_MAX_PEERS                                              */
  int64_t out_peer_words; /* TBS_OUT_PEERS: uint64 words of EVERY out_peers buffer; must equal
                             nbuckets (SDH) or 1 (2PCF), else TBS_EINVAL                    */
} tbs_args;
#define TBS_MAX_PEERS 16

int tbs_sdh_ex(const tbs_args* args, float bucket_width, int nbuckets, uint64_t* hist);
int tbs_pcf_ex(const tbs_args* args, float radius, uint64_t* count);
int tbs_pairmatrix_ex(const tbs_args* args, tbs_kernel kernel, float* out);

/* ---- NEXT rows ---------------------------------------------------- */

/* Kernel-density pair sum, a Type-I 2-BS ("Kernel density/regression"):
 * *sum = sum_{i<j} exp(-gamma * ||p_i - p_j||^2) over points[n][3], host or device pointers,
 * synchronous. fp32 kernel values, fp32 Kahan per thread, fp64 across threads; the CTA
 * partials are combined with fp64 atomics, so the last bits can differ run to run. */
int tbs_kde(const float* points, int64_t n, float gamma, double* sum);
int tbs_kde_ex(const tbs_args* args, float gamma, double* sum);   /* sum: device, overwritten */

/* All-point k-nearest neighbours, a Type-I 2-BS ("all-point k-nearest
 * neighbors (when k is small)"; reading R5). For every anchor i (all i in [0, n) for
 * tbs_knn; i in [row_begin, row_end) for tbs_knn_ex), the k points j != i of smallest Euclidean
 * distance, ascending by (fp32 squared distance, j): equal distances list the smaller index
 * first. Row r = i - row_begin: idx[r*k + t] (int32, j) and dist[r*k + t] (fp32, the correctly
 * rounded sqrt of the fp32 squared distance), t = 0..k-1; if n - 1 < k the missing entries are
 * idx -1, dist +inf. 1 <= k <= TBS_KNN_MAX_K; coordinates must be finite.
 * tbs_knn: points[n][dim] and idx/dist host or device (all alike), synchronous.
 * tbs_knn_ex: device pointers, enqueued on args->stream; ev_begin/ev_end bracket the kNN
 * kernel and its segment merge. Scratch is stream-ordered and freed on return. */
#define TBS_KNN_MAX_K 32
int tbs_knn(const float* points, int64_t n, int dim, int k, int32_t* idx, float* dist);
int tbs_knn_ex(const tbs_args* args, int k, int32_t* idx, float* dist);

/* Radial distribution function, "a normalized form of SDH" (§III-B; DESIGN.md
 * reading R6). For the nb real shells k w <= d < (k+1) w, k = 0..nb-1:
 *   g[k] = h[k] / (P * shell_k / volume),  shell_k = c_dim (((k+1) w)^dim - (k w)^dim),
 * c_dim the unit dim-ball volume (no periodic boundary), h the SDH of the same pairs computed
 * with nb+1 buckets (bucket nb holds every d >= nb w and is not a shell, so it is dropped) and
 * P the number of pairs h counts: sum over the anchor rows i in [row_begin, row_end) of
 * (n - 1 - i) (C(n,2) for the whole set). g: fp64 [nb], overwritten. TBS_EXACT_LATTICE and the
 * SDH's other flags apply to the histogram (TBS_OUT_PEERS: TBS_EUNSUPPORTED, use
 * tbs_rdf_hist_ex on the combined histogram). volume must be finite and > 0.
 * tbs_rdf: host or device pointers, synchronous. tbs_rdf_ex: device pointers, enqueued. */
int tbs_rdf(const float* points, int64_t n, int dim, float bucket_width, int nbuckets, double volume, double* g);
int tbs_rdf_ex(const tbs_args* args, float bucket_width, int nbuckets, double volume, double* g);
/* The normalisation alone, on the device, for a histogram combined across ranks: hist is a
 * device uint64 [>= nbuckets] (its first nbuckets real shells are used), pairs the pairs it
 * counts (n(n-1)/2 after the all-reduce), g a device fp64 [nbuckets]; enqueued on `stream`. */
int tbs_rdf_hist_ex(const uint64_t* hist, int nbuckets, int dim, float bucket_width, double pairs, double volume,
                    double* g, void* stream);

/* High-dimensional Type-III pair matrix on the 5th-generation tensor cores (NEXT-3;
 * PAPER.md L330-332 kernel methods over feature spaces): features are bf16 [n][d] row-major
 * (raw 16-bit patterns), 1 <= d <= 1024 (larger d: TBS_EUNSUPPORTED). out[i*n + j] = K(x_i, x_j)
 * in fp32 for all i, j (diagonal included) with s = |x_i|^2 + |x_j|^2 - 2 x_i.x_j from
 * tcgen05 bf16 x bf16 -> fp32 dot products (error ~2^-22 (|x_i|^2 + |x_j|^2) on s), clamped
 * at 0 for the distance kernels. Host or device pointers, synchronous. */
int tbs_pairmatrix_hd(const uint16_t* features, int64_t n, int d, tbs_kernel kernel, float* out);
/* Device pointers, rows [row_begin, row_end) x n into out, enqueued on `stream`; optional
 * cudaEvent_t pair recorded around the tensor-core kernel. */
int tbs_pairmatrix_hd_ex(const uint16_t* features, int64_t n, int d, int64_t row_begin, int64_t row_end,
                         tbs_kernel kernel, float* out, void* stream, void* ev_begin, void* ev_end);

/* Pair-count-balanced anchor-row partition for multi-GPU: rank r of
 * `world` gets [*row_begin, *row_end) such that sum over its rows of (n-1-i) is
 * n(n-1)/(2*world) up to one row; the ranges are disjoint and cover [0, n). Host-only. */
int tbs_rank_rows(int64_t n, int world, int rank, int64_t* row_begin, int64_t* row_end);

/* Plumbing of the fused combine (host-only, CUDA IPC; TBS_OUT_PEERS). tbs_peer_alloc makes a
 * zeroed device buffer of `bytes` on the current device (its own cudaMalloc allocation, so
 * the IPC mapping starts at offset 0) and writes its 64-byte IPC handle to `handle`;
 * tbs_peer_open maps another process's buffer from its handle (peer access over NVLink is
 * enabled by the mapping); tbs_peer_close unmaps; tbs_peer_free frees an own buffer. */
int tbs_peer_alloc(uint64_t bytes, void** dev_ptr, void* handle);
int tbs_peer_open(const void* handle, void** dev_ptr);
int tbs_peer_close(void* dev_ptr);
int tbs_peer_free(void* dev_ptr);
/* *ok = 1 if the current device can add into memory of the GPU with PCI bus id `pci_bus_id`
 * ("dddd:bb:dd.f") with native atomics (same device, or peer access with
 * cudaDevP2PAttrNativeAtomicSupported); 0 otherwise, including a GPU this process cannot see.
 * The fused combine relies on system-scope atomics over peer memory: without native support
 * (e.g. PCIe P2P) the adds are not atomic, so callers must fall back to the all-reduce. */
int tbs_peer_atomics_ok(const char* pci_bus_id, int* ok);

/* Thread-local text of the last non-OK status ("" if none). */
const char* tbs_last_error(void);

/* Trim the cached scratch of the current device's default memory pool. */
void tbs_release(void);

/* Number of kernels this library has launched in this process (evidence counter). */
uint64_t tbs_launch_count(void);

/* ABI version (major * 100 + minor). */
int tbs_version(void);

#ifdef __cplusplus
}
#endif
#endif /* TBS_H_ */
