// rotation.cuh -- the Jacobi rotation of eq (4), shared by the one-sided kernels
// (pairs of columns a_i, a_j) and the two-sided EVD (pairs of indices of a symmetric B, PAPER.md:97-99;
// same formula with alpha = b_ii, beta = b_jj, gamma = b_ij).
#pragma once

namespace wcsvd {

// Threshold test and rotation for squared norms alpha, beta >= 0 and dot product
// gamma, with tol2 = tol^2: rotate iff alpha, beta > 0 and gamma^2 > tol^2 alpha beta
// (<=> |gamma| > tol sqrt(alpha) sqrt(beta); inputs are pre-scaled to max|a_ij| < 1 so the products
// cannot overflow; a product that underflows to 0 means a numerically zero column: no rotation).
// tau = (alpha - beta)/(2 gamma), t = sgn(tau)/(|tau| + sqrt(1 + tau^2)) is evaluated as
// t = sgn(tau) 2|gamma| / (|d| + sqrt(d^2 + 4 gamma^2)), d = alpha - beta: the same number, multiplied
// through by 2|gamma|, with one correctly-rounded reciprocal instead of three divisions.
// sgn(0) = +1 (Z4). c = 1/sqrt(1 + t^2), s = t c. Returns true (c, s, t) if the pair rotates.
__device__ __forceinline__ bool jacobi_rotation(double alpha, double beta, double gamma, double tol2,
                                                double& c, double& s, double& t) {
  c = 1.0;
  s = 0.0;
  t = 0.0;
  const double ab = alpha * beta;
  if (!(ab > 0.0) || gamma * gamma <= tol2 * ab) return false;
  const double d = alpha - beta;
  const double r = sqrt(fma(d, d, 4.0 * (gamma * gamma)));
  const double sg = (d == 0.0 || ((d > 0.0) == (gamma > 0.0))) ? 1.0 : -1.0;
  t = (sg * 2.0 * fabs(gamma)) * __drcp_rn(fabs(d) + r);
  c = rsqrt(fma(t, t, 1.0));
  s = t * c;
  return true;
}

}  // namespace wcsvd
