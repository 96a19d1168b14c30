// complete.cu -- deterministic completion of U for (numerically) zero singular values.
//
// PAPER.md:181 (§III.C): once V is known, U and Sigma are "easily deduced" as u_j = a_j / sigma_j.
// That breaks down for sigma_j ~ 0 (rank deficiency). Finalisation writes such columns as signed
// zeros (the sign is the Z15 flip of the matching v_j) and flags the matrix; this pass replaces
// each one, in rank order, by the unit vector e_i farthest from the span of all previous columns
// (largest residual^2 = 1 - sum_q u_q[i]^2, first i on ties; DESIGN.md §3 Z14 -- the largest is
// >= (M-k)/M, so it always exists), orthogonalised against them by modified Gram-Schmidt,
// normalised and signed. Rare path: only flagged matrices do work. One CTA per matrix; row sums in
// a fixed order and fixed-order block reductions (deterministic).
#include <cuda_runtime.h>

#include "common.cuh"
#include "kernels.h"

namespace wcsvd {

namespace {

constexpr int kCT = 256;

__device__ double block_sum(double v, double* red) {
  for (int off = 16; off > 0; off >>= 1) v += __shfl_xor_sync(0xffffffffu, v, off);
  const int w = threadIdx.x >> 5, l = threadIdx.x & 31;
  __syncthreads();
  if (l == 0) red[w] = v;
  __syncthreads();
  double s = 0.0;
  for (int i = 0; i < kCT / 32; ++i) s += red[i];  // fixed order, every thread
  return s;
}

}  // namespace

template <typename TI>
__global__ void __launch_bounds__(kCT) complete_u_kernel(const MatDesc* __restrict__ descs, int count) {
  const MatDesc d = descs[blockIdx.x];
  if (!d.status || !(d.status[d.idx] & kNeedsCompletion)) return;
  TI* Uw = reinterpret_cast<TI*>(d.swapped ? d.V : d.U);  // X-space left factor (M x N, ld ldW)
  const TI* S = reinterpret_cast<const TI*>(d.S);
  const int ld = d.swapped ? d.ldv : d.ldu;
  if (!Uw) return;
  const int M = d.M, N = d.N;
  __shared__ double x[1024];
  __shared__ double red[kCT / 32];
  __shared__ double s_res[kCT / 32];
  __shared__ int s_idx[kCT / 32];
  (void)S;
  for (int k = 0; k < N; ++k) {
    // Complete exactly the columns finalisation wrote as (signed) zeros: the finalising kernel applied
    // its own rank threshold (sigma_1 M 2^-53 on the fp64 iterate, 2^-24 for the fp32 Level-0 kernel),
    // so this pass never overwrites a valid column (a unit vector is never all zero).
    int nz = 0;
    for (int r = threadIdx.x; r < M; r += kCT) nz |= ((double)Uw[(size_t)k * ld + r] != 0.0);
    if (__syncthreads_or(nz)) continue;
    const double sgn = signbit((double)Uw[(size_t)k * ld]) ? -1.0 : 1.0;  // Z15 flip recorded as -0.0
    // candidate e_i with the largest residual^2 = 1 - sum_{q<k} u_q[i]^2 (first i on ties)
    double bres = -1.0;
    int bidx = 0x7fffffff;
    for (int r = threadIdx.x; r < M; r += kCT) {
      double p2 = 0.0;
      for (int q = 0; q < k; ++q) {
        const double u = (double)Uw[(size_t)q * ld + r];
        p2 = fma(u, u, p2);
      }
      const double res2 = 1.0 - p2;
      if (res2 > bres) { bres = res2; bidx = r; }  // r ascending per thread: first on ties
    }
    for (int off = 16; off > 0; off >>= 1) {
      const double ob = __shfl_xor_sync(0xffffffffu, bres, off);
      const int oi = __shfl_xor_sync(0xffffffffu, bidx, off);
      if (ob > bres || (ob == bres && oi < bidx)) { bres = ob; bidx = oi; }
    }
    __syncthreads();
    if ((threadIdx.x & 31) == 0) { s_res[threadIdx.x >> 5] = bres; s_idx[threadIdx.x >> 5] = bidx; }
    __syncthreads();
    int best = s_idx[0];
    double bb = s_res[0];
    for (int w = 1; w < kCT / 32; ++w)
      if (s_res[w] > bb || (s_res[w] == bb && s_idx[w] < best)) { bb = s_res[w]; best = s_idx[w]; }
    for (int r = threadIdx.x; r < M; r += kCT) x[r] = (r == best) ? 1.0 : 0.0;
    __syncthreads();
    for (int q = 0; q < k; ++q) {
      const TI* uq = Uw + (size_t)q * ld;
      double p = 0.0;
      for (int r = threadIdx.x; r < M; r += kCT) p = fma((double)uq[r], x[r], p);
      p = block_sum(p, red);
      for (int r = threadIdx.x; r < M; r += kCT) x[r] = fma(-p, (double)uq[r], x[r]);
      __syncthreads();
    }
    double nn = 0.0;
    for (int r = threadIdx.x; r < M; r += kCT) nn = fma(x[r], x[r], nn);
    const double res = sqrt(block_sum(nn, red));
    for (int r = threadIdx.x; r < M; r += kCT) Uw[(size_t)k * ld + r] = (TI)(sgn * (x[r] / res));
    __syncthreads();
  }
  (void)count;
}

cudaError_t launch_complete(int fp32, const MatDesc* descs, int count, cudaStream_t stream) {
  if (count <= 0) return cudaSuccess;
  if (fp32)
    complete_u_kernel<float><<<count, kCT, 0, stream>>>(descs, count);
  else
    complete_u_kernel<double><<<count, kCT, 0, stream>>>(descs, count);
  return cudaGetLastError();
}

}  // namespace wcsvd
