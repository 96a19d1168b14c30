// rotation.cuh -- the Jacobi rotation of eq (4), shared by the one-sided kernels
// (pairs of columns a_i, a_j) and the two-sided EVD (pairs of indices of a symmetric B, PAPER.md:97-99;
// same formula with alpha = b_ii, beta = b_jj, gamma = b_ij).
#pragma once

namespace wcsvd {

// Threshold test and rotation for squared norms alpha, beta >= 0 and dot product
// gamma, with tol2 = tol^2: rotate iff alpha, beta > 0 and gamma^2 > tol^2 alpha beta
// (<=> |gamma| > tol sqrt(alpha) sqrt(beta); inputs are pre-scaled to max|a_ij| < 1 so the products
// cannot overflow; a product that underflows to 0 means a numerically zero column: no rotation).
// eq (4): tau = (alpha - beta)/(2 gamma), t = sgn(tau)/(|tau| + sqrt(1 + tau^2)), c = 1/sqrt(1+t^2),
// s = t c, sgn(0) = +1 (Z4). Evaluated without divisions (R-ROT): with d = alpha - beta,
// r = sqrt(d^2 + 4 gamma^2) and q = 1/sqrt(2 r (r + |d|)):
//   c = (r + |d|) q,   s = sgn(tau) 2|gamma| q,   t = s / c = sgn(tau) 4 r |gamma| q^2,
// the same numbers as eq (4) (multiply num/denom of t by 2|gamma|; 1/(r+|d|) = 2 r q^2), with one
// sqrt and one rsqrt on the dependent chain. Returns true (c, s, t) if the pair rotates.
__device__ __forceinline__ bool jacobi_rotation(double alpha, double beta, double gamma, double tol2,
                                                double& c, double& s, double& t) {
  c = 1.0;
  s = 0.0;
  t = 0.0;
  const double ab = alpha * beta;
  const double g2 = gamma * gamma;
  if (!(ab > 0.0) || g2 <= tol2 * ab) return false;
  const double d = alpha - beta, ad = fabs(d);
  const double r = sqrt(fma(d, d, 4.0 * g2));
  const double rp = r + ad;
  const double q = rsqrt(2.0 * r * rp);
  const double sg = (d == 0.0 || ((d > 0.0) == (gamma > 0.0))) ? 2.0 : -2.0;  // 2 sgn(tau)
  const double sq = sg * fabs(gamma) * q;  // s
  c = rp * q;
  s = sq;
  t = 2.0 * r * sq * q;  // sgn(tau) 4 r |gamma| q^2
  return true;
}

// fp32 variant of the same evaluation (wcsvd_batched_f32, Level 0).
__device__ __forceinline__ bool jacobi_rotation(float alpha, float beta, float gamma, float tol2, float& c,
                                                float& s, float& t) {
  c = 1.0f;
  s = 0.0f;
  t = 0.0f;
  const float ab = alpha * beta;
  const float g2 = gamma * gamma;
  if (!(ab > 0.0f) || g2 <= tol2 * ab) return false;
  const float d = alpha - beta, ad = fabsf(d);
  const float r = sqrtf(fmaf(d, d, 4.0f * g2));
  const float rp = r + ad;
  const float q = rsqrtf(2.0f * r * rp);
  const float sg = (d == 0.0f || ((d > 0.0f) == (gamma > 0.0f))) ? 2.0f : -2.0f;
  const float sq = sg * fabsf(gamma) * q;
  c = rp * q;
  s = sq;
  t = 2.0f * r * sq * q;
  return true;
}

// Same rotation with the angle evaluated in fp32 (R-ROT32). The threshold test and d
// are fp64; (d, gamma) are rescaled by an exact power of two into fp32 range (t is homogeneous of
// degree 0 in them), t is formed in fp32 (~1e-7 relative), then c = 1/sqrt(1 + t^2) and s = t c are
// fp64, so the rotation applied is orthogonal to fp64 rounding; only its angle differs from the
// exact eq (4) angle by ~1e-7 relative, which changes the pace of convergence, not the result.
// Updates that follow must use the general forms valid for any (c, s) (eq 6 as printed; the full
// 2x2 two-sided update), not the closed forms that assume the exact angle.
__device__ __forceinline__ bool jacobi_rotation_f32(double alpha, double beta, double gamma, double tol2,
                                                    double& c, double& s) {
  c = 1.0;
  s = 0.0;
  const double ab = alpha * beta;
  const double g2 = gamma * gamma;
  if (!(ab > 0.0) || g2 <= tol2 * ab) return false;
  const double d = alpha - beta;
  const double mx = fmax(fabs(d), fabs(gamma));
  const int ex = (int)((unsigned long long)__double_as_longlong(mx) >> 52) & 0x7ff;  // mx > 0, normal
  const double sc = __longlong_as_double((long long)(2046 - ex) << 52);              // 2^-(ex-1023)
  const float df = __double2float_rn(d * sc), gf = __double2float_rn(gamma * sc);
  const float r = sqrtf(fmaf(df, df, 4.0f * gf * gf));
  const float sg = (df == 0.0f || ((df > 0.0f) == (gf > 0.0f))) ? 2.0f : -2.0f;
  const double t = (double)(sg * fabsf(gf) * __frcp_rn(fabsf(df) + r));
  c = rsqrt(fma(t, t, 1.0));
  s = t * c;
  return true;
}

}  // namespace wcsvd
