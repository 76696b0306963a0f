// tbs_rdf.cuh — radial distribution function epilogue (NEXT-1): the SDH's ideal-gas
// normalisation, "a normalized form of SDH" (§III-B; reading R6).
//
//   g[k] = h[k] / (P * V_shell(k) / volume),  V_shell(k) = V_dim((k+1) w) - V_dim(k w)
//
// derived here independently of the test-side reference: the dim-ball volume V_d(r) = c_d r^d with the
// unit-ball constants from the recursion c_0 = 1, c_1 = 2, c_d = c_{d-2} * 2 pi / d, and the
// shell written as c_d w^d ((k+1)^d - k^d) with the bracket expanded by the binomial theorem,
// sum_{i<d} C(d, i) k^i (Horner), so no two large powers are subtracted at large k.
#pragma once
#include <cstdint>

namespace tbs {

__global__ void rdf_kernel(const unsigned long long* __restrict__ hist, int nb, int dim, double w, double pairs,
                           double volume, double* __restrict__ g) {
  double c = (dim & 1) ? 2.0 : 1.0;
  for (int d = (dim & 1) ? 3 : 2; d <= dim; d += 2) c *= 2.0 * 3.141592653589793238462643 / (double)d;
  double wd = 1.0;
  for (int d = 0; d < dim; ++d) wd *= w;
  double binom[5] = {1.0, 0.0, 0.0, 0.0, 0.0};   // row `dim` of Pascal's triangle
  for (int r = 1; r <= dim; ++r)
    for (int i = r; i >= 1; --i) binom[i] += binom[i - 1];
  const double scale = pairs * c * wd / volume;
  for (int k = blockIdx.x * blockDim.x + threadIdx.x; k < nb; k += gridDim.x * blockDim.x) {
    const double kk = (double)k;
    double diff = 0.0;                             // (k+1)^dim - k^dim = sum_{i<dim} C(dim,i) k^i
    for (int i = dim - 1; i >= 0; --i) diff = diff * kk + binom[i];
    const double ideal = scale * diff;
    g[k] = ideal > 0.0 ? (double)hist[k] / ideal : 0.0;
  }
}

}  // namespace tbs
