/*
 * tbs_oracle.c — the CPU ORACLE for the 2-body-statistics hot path.
 *
 * TEST INFRASTRUCTURE ONLY. Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs may load this library. The product path
 * (paper_conf_icpp_pitaksirianannt16_b200/, libtbs.so) never links, imports or
 * calls it, and shares no source, header, helper or constant with it.
 *
 * What it computes: the plain definitions of the three 2-BS outputs, evaluated
 * pair by pair in double precision from the fp32 input coordinates (which convert
 * to double exactly). Citations are to /root/reference/PAPER.md lines (L<a>-<b>).
 *
 *  - Pair semantics: every unordered pair {i, j}, i < j, exactly once; no
 *    self-pairs. Alg. 1 loops i = t+1 .. N (L290-296); Alg. 2 covers inter-block
 *    i > b and intra-block i > t (L436-458).
 *  - Distance function: Euclidean distance (L600-602 "pairwise Euclidean
 *    distances"; L841-843 for SDH).
 *  - SDH (Type-II): "a histogram that shows the distribution of all distances
 *    computed" (L841-847); Alg. 3 line 7 increments SHMOut[d] with d the bucket
 *    of the distance (L496-511). Readings: half-open buckets
 *    [k w, (k+1) w) (Q1) and distances >= nb*w clamped into bucket nb-1 (Q2).
 *  - 2PCF (Type-I): "one scalar describing the number of points within a radius"
 *    (L600-604); reading Q4: unordered pairs with d < r.
 *  - Type-III: "kernel functions for all pairs of data" (L330-332); reading Q10:
 *    Gaussian exp(-gamma * ||x - y||^2), full n x n including the diagonal.
 *  - OpenMP structure mirrors the paper's CPU baseline: private per-thread
 *    histograms merged at the end (L868-872), schedule(guided) (L909-912).
 *
 * No SIMD intrinsics, no blocking, no reordering beyond the definition. Compile
 * with -O2 -ffp-contract=off -fopenmp.
 *
 * Row-range variant: every function takes [row_begin, row_end): only anchors i in
 * that range contribute, each with all partners j > i.
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <omp.h>

#define ORACLE_OK 0
#define ORACLE_EINVAL 1
#define ORACLE_ENOMEM 2

int oracle_num_threads(void) { return omp_get_max_threads(); }

/* Squared Euclidean distance in double (L600-602). */
static double dist2(const float* P, int dim, int64_t i, int64_t j) {
  double s = 0.0;
  for (int c = 0; c < dim; ++c) {
    double d = (double)P[i * dim + c] - (double)P[j * dim + c];
    s += d * d;
  }
  return s;
}

static int check_common(const float* P, int64_t n, int dim, int64_t rb, int64_t re) {
  if (n < 0 || dim < 1 || dim > 4) return ORACLE_EINVAL;
  if (rb < 0 || re < rb || re > n) return ORACLE_EINVAL;
  if (n >= 2 && P == NULL) return ORACLE_EINVAL;
  return ORACLE_OK;
}

/*
 * SDH, float mode. hist[b] = #{i<j : min(floor(d_ij / w), nb-1) = b}.
 * amb (optional, length nb+1): amb[e] = #{i<j : |d_ij - e w| <= 1e-6 e w},
 * e = 1..nb-1 — the pairs whose bucket an fp32 evaluation may legitimately
 * place on either side of edge e (acceptance rule).
 * amb_diag (optional, length nb+1): the same count for the narrower 5e-7 band,
 * the diagnostic SURVEY §8(c) asks to report beside the 1e-6 rule ("also report,
 * as a diagnostic, the mismatch count against a 5e-7 band").
 * w is the caller's fp32 bucket width, passed already widened to double.
 */
int oracle_sdh_bands(const float* P, int64_t n, int dim, double w, int nb,
                     int64_t row_begin, int64_t row_end, uint64_t* hist, uint64_t* amb, uint64_t* amb_diag) {
  if (check_common(P, n, dim, row_begin, row_end) || nb < 1 || !(w > 0.0) || isinf(w) || !hist)
    return ORACLE_EINVAL;
  int T = omp_get_max_threads();
  uint64_t* ph = (uint64_t*)calloc((size_t)T * nb, sizeof(uint64_t));
  uint64_t* pa = (uint64_t*)calloc((size_t)T * (nb + 1), sizeof(uint64_t));
  uint64_t* pd = (uint64_t*)calloc((size_t)T * (nb + 1), sizeof(uint64_t));
  if (!ph || !pa || !pd) { free(ph); free(pa); free(pd); return ORACLE_ENOMEM; }
#pragma omp parallel
  {
    uint64_t* h = ph + (size_t)omp_get_thread_num() * nb;
    uint64_t* a = pa + (size_t)omp_get_thread_num() * (nb + 1);
    uint64_t* a2 = pd + (size_t)omp_get_thread_num() * (nb + 1);
#pragma omp for schedule(guided)
    for (int64_t i = row_begin; i < row_end; ++i) {
      for (int64_t j = i + 1; j < n; ++j) {
        double d = sqrt(dist2(P, dim, i, j));
        double q = d / w;
        int b = (q >= (double)nb) ? nb - 1 : (int)floor(q);
        h[b] += 1;
        double e = rint(q);
        if (e >= 1.0 && e <= (double)(nb - 1) && fabs(d - e * w) <= 1e-6 * e * w) a[(int)e] += 1;
        if (e >= 1.0 && e <= (double)(nb - 1) && fabs(d - e * w) <= 5e-7 * e * w) a2[(int)e] += 1;
      }
    }
  }
  memset(hist, 0, sizeof(uint64_t) * nb);
  if (amb) memset(amb, 0, sizeof(uint64_t) * (nb + 1));
  if (amb_diag) memset(amb_diag, 0, sizeof(uint64_t) * (nb + 1));
  for (int t = 0; t < T; ++t) {
    for (int b = 0; b < nb; ++b) hist[b] += ph[(size_t)t * nb + b];
    if (amb) for (int e = 0; e <= nb; ++e) amb[e] += pa[(size_t)t * (nb + 1) + e];
    if (amb_diag) for (int e = 0; e <= nb; ++e) amb_diag[e] += pd[(size_t)t * (nb + 1) + e];
  }
  free(ph); free(pa); free(pd);
  return ORACLE_OK;
}

int oracle_sdh(const float* P, int64_t n, int dim, double w, int nb,
               int64_t row_begin, int64_t row_end, uint64_t* hist, uint64_t* amb) {
  return oracle_sdh_bands(P, n, dim, w, nb, row_begin, row_end, hist, amb, NULL);
}

/* Exact integer square root: largest r with r*r <= S, for 0 <= S < 2^62. */
static int64_t isqrt64(int64_t S) {
  int64_t r = (int64_t)sqrt((double)S);
  while (r > 0 && r * r > S) --r;
  while ((r + 1) * (r + 1) <= S) ++r;
  return r;
}

/*
 * SDH, exact-lattice mode (BASELINE.json north star: "exact integer
 * squared-distance bucketing"). Coordinates must be integer-valued; the bucket
 * width is dyadic, w = m * 2^-j. With s = sum (dx)^2 as an integer,
 *   bucket = min(floor(isqrt(4^j s) / m), nb - 1) = max{k : (k w)^2 <= s} clamped,
 * which is the float-mode definition floor(d / w) evaluated exactly (ties at an
 * edge go to the upper bucket, reading Q1).
 */
int oracle_sdh_lattice(const float* P, int64_t n, int dim, int64_t m, int j2, int nb,
                       int64_t row_begin, int64_t row_end, uint64_t* hist) {
  if (check_common(P, n, dim, row_begin, row_end) || nb < 1 || m < 1 || j2 < 0 || j2 > 30 || !hist)
    return ORACLE_EINVAL;
  for (int64_t i = 0; i < n * dim; ++i) {
    float v = P[i];
    if (v != floorf(v) || fabsf(v) > 16777216.0f) return ORACLE_EINVAL;
  }
  int T = omp_get_max_threads();
  uint64_t* ph = (uint64_t*)calloc((size_t)T * nb, sizeof(uint64_t));
  if (!ph) return ORACLE_ENOMEM;
  int bad = 0;
#pragma omp parallel reduction(|: bad)
  {
    uint64_t* h = ph + (size_t)omp_get_thread_num() * nb;
#pragma omp for schedule(guided)
    for (int64_t i = row_begin; i < row_end; ++i) {
      for (int64_t jj = i + 1; jj < n; ++jj) {
        int64_t s = 0;
        for (int c = 0; c < dim; ++c) {
          int64_t d = (int64_t)P[i * dim + c] - (int64_t)P[jj * dim + c];
          s += d * d;
        }
        if (s > ((int64_t)1 << (62 - 2 * j2))) { bad = 1; continue; }
        int64_t k = isqrt64(s << (2 * j2)) / m;
        if (k > nb - 1) k = nb - 1;
        h[k] += 1;
      }
    }
  }
  memset(hist, 0, sizeof(uint64_t) * nb);
  for (int t = 0; t < T; ++t)
    for (int b = 0; b < nb; ++b) hist[b] += ph[(size_t)t * nb + b];
  free(ph);
  return bad ? ORACLE_EINVAL : ORACLE_OK;
}

/*
 * 2PCF: count = #{i<j : d_ij < r} (L600-604, reading Q4).
 * amb (optional): #{i<j : |d_ij - r| <= 1e-6 r}.
 */
int oracle_pcf(const float* P, int64_t n, int dim, double r, int64_t row_begin, int64_t row_end,
               uint64_t* count, uint64_t* amb) {
  if (check_common(P, n, dim, row_begin, row_end) || !(r >= 0.0) || !count) return ORACLE_EINVAL;
  uint64_t c = 0, a = 0;
#pragma omp parallel for schedule(guided) reduction(+: c, a)
  for (int64_t i = row_begin; i < row_end; ++i) {
    for (int64_t j = i + 1; j < n; ++j) {
      double d = sqrt(dist2(P, dim, i, j));
      if (d < r) c += 1;
      if (fabs(d - r) <= 1e-6 * r) a += 1;
    }
  }
  *count = c;
  if (amb) *amb = a;
  return ORACLE_OK;
}

/*
 * Type-III pairwise-kernel matrix (L323-332, L709-712; reading Q10):
 * out[(i - row_begin) * n + j] = K(p_i, p_j) for i in [row_begin, row_end), all j in
 * [0, n) (diagonal included), with K selected by ktype as in include/tbs.h:
 *   0 Gaussian exp(-gamma * ||p_i - p_j||^2), 1 squared distance, 2 distance.
 */
int oracle_pairmatrix(const float* P, int64_t n, int dim, int ktype, double gamma, int64_t row_begin,
                      int64_t row_end, double* out) {
  if (check_common(P, n, dim, row_begin, row_end) || !isfinite(gamma) || ktype < 0 || ktype > 2)
    return ORACLE_EINVAL;
  if (row_end > row_begin && !out) return ORACLE_EINVAL;
#pragma omp parallel for schedule(guided)
  for (int64_t i = row_begin; i < row_end; ++i)
    for (int64_t j = 0; j < n; ++j) {
      double s = dist2(P, dim, i, j);
      out[(i - row_begin) * n + j] = ktype == 0 ? exp(-gamma * s) : ktype == 1 ? s : sqrt(s);
    }
  return ORACLE_OK;
}

/*
 * Closed form of the lattice SDH for the full cubic lattice {0..L-1}^3 (any
 * permutation of its points), O(L^3). For displacement (dx, dy, dz) the number of
 * ordered point pairs is prod_c (L - |d_c|); folding the sign of each axis,
 *   hist[k] = 1/2 * sum_{(a,b,c) in [0,L)^3 \ 0} mu(a) mu(b) mu(c) [bucket(a^2+b^2+c^2) = k],
 *   mu(a) = (L - a) * (a > 0 ? 2 : 1),
 * with the same exact dyadic bucketing as oracle_sdh_lattice. A second, O(L^3)
 * route to the same numbers (pinned against the brute-force oracle in tests), used
 * for parity at lattice sizes where the O(N^2) loop would take hours.
 * If r2 >= 0, *count_lt additionally receives #{pairs : s < r2} (2PCF on the lattice).
 */
int oracle_lattice_closed(int64_t L, int64_t m, int j2, int nb, uint64_t* hist, int64_t r2,
                          uint64_t* count_lt) {
  if (L < 1 || m < 1 || j2 < 0 || j2 > 30 || nb < 1 || !hist) return ORACLE_EINVAL;
  if (3 * (L - 1) * (L - 1) > ((int64_t)1 << (62 - 2 * j2))) return ORACLE_EINVAL;
  /* twice the answer accumulates in unsigned 64-bit; halve at the end */
  uint64_t* h2 = (uint64_t*)calloc((size_t)nb, sizeof(uint64_t));
  if (!h2) return ORACLE_ENOMEM;
  uint64_t c2 = 0;
  for (int64_t a = 0; a < L; ++a)
    for (int64_t b = 0; b < L; ++b)
      for (int64_t c = 0; c < L; ++c) {
        if (a == 0 && b == 0 && c == 0) continue;
        uint64_t mu = (uint64_t)((L - a) * (a > 0 ? 2 : 1)) * (uint64_t)((L - b) * (b > 0 ? 2 : 1)) *
                      (uint64_t)((L - c) * (c > 0 ? 2 : 1));
        int64_t s = a * a + b * b + c * c;
        int64_t k = isqrt64(s << (2 * j2)) / m;
        if (k > nb - 1) k = nb - 1;
        h2[k] += mu;
        if (r2 >= 0 && s < r2) c2 += mu;
      }
  for (int k = 0; k < nb; ++k) hist[k] = h2[k] / 2;
  if (count_lt) *count_lt = c2 / 2;
  free(h2);
  return ORACLE_OK;
}

/*
 * Kernel-density pair sum (Type-I, NEXT-2 of SURVEY §8(f); PAPER.md L303-314 names
 * "Kernel density/regression" as a Type-I 2-BS whose per-thread output fits in
 * registers): S = sum_{i<j} exp(-gamma * ||p_i - p_j||^2), Gaussian kernel (reading Q10's
 * kernel). Row-range variant as above. Plain double accumulation per thread, merged.
 */
int oracle_kde(const float* P, int64_t n, int dim, double gamma, int64_t row_begin, int64_t row_end,
               double* sum) {
  if (check_common(P, n, dim, row_begin, row_end) || !isfinite(gamma) || !sum) return ORACLE_EINVAL;
  double acc = 0.0;
#pragma omp parallel for schedule(guided) reduction(+: acc)
  for (int64_t i = row_begin; i < row_end; ++i)
    for (int64_t j = i + 1; j < n; ++j) acc += exp(-gamma * dist2(P, dim, i, j));
  *sum = acc;
  return ORACLE_OK;
}

/*
 * Radial distribution function (Type-II, NEXT-1; "RDF, which outputs a
 * normalized form of SDH"): g[k] = hist[k] / ideal[k], k = 0..nb-1, with ideal[k] the
 * expected count of an ideal gas over the same pairs in volume V,
 *   ideal[k] = pairs * shell_k / V,   shell_k = vol of the dim-ball shell k w <= r < (k+1) w
 *            = c_dim ((k+1) w)^dim - c_dim (k w)^dim,
 * unit-ball volumes c_1..c_4 = 2, pi, 4 pi / 3, pi^2 / 2. Reading R6: hist holds
 * the counts of the nb real shells only (an SDH with nb+1 buckets whose clamp bucket nb is
 * dropped), and `pairs` is the number of pairs that histogram counted (C(n,2) for the whole
 * set, sum_{i in [b,e)} (n-1-i) for an anchor-row range).
 */
int oracle_rdf(const uint64_t* hist, int nb, int dim, double w, double pairs, double volume, double* g) {
  if (!hist || !g || nb < 1 || dim < 1 || dim > 4 || !(w > 0.0) || !(volume > 0.0) || !(pairs >= 0.0))
    return ORACLE_EINVAL;
  static const double unit_ball[5] = {0.0, 2.0, 3.14159265358979323846, 4.18879020478639098462,
                                      4.93480220054467930942};
  for (int k = 0; k < nb; ++k) {
    const double shell = unit_ball[dim] * (pow((k + 1) * w, dim) - pow(k * w, dim));
    const double ideal = pairs * shell / volume;
    g[k] = ideal > 0.0 ? (double)hist[k] / ideal : 0.0;
  }
  return ORACLE_OK;
}

/* bf16 bit pattern -> float (exact: bf16 is the top half of an fp32). */
static double bf16_to_double(uint16_t h) {
  uint32_t u = (uint32_t)h << 16;
  float f;
  memcpy(&f, &u, 4);
  return (double)f;
}

/*
 * High-dimensional Type-III pair matrix (NEXT-3 of SURVEY §8(f); "Kernel
 * methods which compute kernel functions for all pairs of data in the feature space"):
 * features are bf16 [n][d] row-major (passed as their 16-bit patterns);
 * out[(i - row_begin) * n + j] = K(x_i, x_j) for i in [row_begin, row_end), j in [0, n), with
 * K as in oracle_pairmatrix (0 Gaussian exp(-gamma s), 1 s, 2 sqrt(s)), s = ||x_i - x_j||^2
 * evaluated directly (difference, then square) in double.
 */
int oracle_pairmatrix_hd(const uint16_t* X, int64_t n, int d, int ktype, double gamma, int64_t row_begin,
                         int64_t row_end, double* out) {
  if (n < 0 || d < 1 || row_begin < 0 || row_end < row_begin || row_end > n || ktype < 0 || ktype > 2 ||
      !isfinite(gamma) || (n > 0 && !X) || (row_end > row_begin && !out))
    return ORACLE_EINVAL;
#pragma omp parallel for schedule(guided)
  for (int64_t i = row_begin; i < row_end; ++i)
    for (int64_t j = 0; j < n; ++j) {
      double s = 0.0;
      for (int c = 0; c < d; ++c) {
        const double t = bf16_to_double(X[i * d + c]) - bf16_to_double(X[j * d + c]);
        s += t * t;
      }
      out[(i - row_begin) * n + j] = ktype == 0 ? exp(-gamma * s) : ktype == 1 ? s : sqrt(s);
    }
  return ORACLE_OK;
}

/*
 * All-point k-nearest neighbours (Type-I, NEXT-2 of SURVEY §8(f); PAPER.md L311-313:
 * "all-point k-nearest neighbors (when k is small)", a Type-I output small enough for
 * registers). For each anchor i in [row_begin, row_end): the k points j != i with the smallest
 * Euclidean distance, in ascending (distance, j) order — equal distances go to the smaller
 * index (reading R5). Written as the definition: scan j = 0 .. n-1, keep the k best so far
 * sorted, and insert a candidate only if it is strictly better than the current k-th (an
 * equal distance never displaces an earlier, smaller index). If n - 1 < k, the missing
 * entries are idx -1, dist +inf. idx/dist are (row_end - row_begin) x k row-major.
 */
int oracle_knn(const float* P, int64_t n, int dim, int k, int64_t row_begin, int64_t row_end, int64_t* idx,
               double* dist) {
  if (check_common(P, n, dim, row_begin, row_end) || k < 1 || (row_end > row_begin && (!idx || !dist)))
    return ORACLE_EINVAL;
  int rc = ORACLE_OK;
#pragma omp parallel
  {
    double* bs = (double*)malloc(sizeof(double) * (size_t)k);
    int64_t* bj = (int64_t*)malloc(sizeof(int64_t) * (size_t)k);
    if (!bs || !bj) {
#pragma omp atomic write
      rc = ORACLE_ENOMEM;
    } else {
#pragma omp for schedule(guided)
      for (int64_t i = row_begin; i < row_end; ++i) {
        for (int t = 0; t < k; ++t) {
          bs[t] = INFINITY;
          bj[t] = -1;
        }
        for (int64_t j = 0; j < n; ++j) {
          if (j == i) continue;
          const double s = dist2(P, dim, i, j);
          if (!(s < bs[k - 1])) continue;
          int t = k - 1;  /* shift worse entries down, insert after every entry <= s */
          while (t > 0 && s < bs[t - 1]) {
            bs[t] = bs[t - 1];
            bj[t] = bj[t - 1];
            --t;
          }
          bs[t] = s;
          bj[t] = j;
        }
        for (int t = 0; t < k; ++t) {
          idx[(i - row_begin) * k + t] = bj[t];
          dist[(i - row_begin) * k + t] = sqrt(bs[t]);
        }
      }
    }
    free(bs);
    free(bj);
  }
  return rc;
}
