// complete.cu -- deterministic completion of U for (numerically) zero singular values.
//
// PAPER.md:181 (§III.C): once V is known, U and Sigma are "easily deduced" as u_j = a_j / sigma_j.
// That breaks down for sigma_j ~ 0 (rank deficiency). Finalisation writes such columns as signed
// zeros (the sign is the Z15 flip of the matching v_j) and flags the matrix; this pass replaces
// each one, in rank order, by the first of e_1, e_2, ... whose modified Gram-Schmidt residual
// against all previous columns exceeds 1/2, normalised and signed. Rare path: only flagged
// matrices do work. One CTA per matrix; fixed-order block reductions (deterministic).
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
  const double eps = sizeof(TI) == 4 ? 5.9604644775390625e-08 : kU53;
  const double thresh = (double)S[0] * (double)M * eps;
  int next_e = 0;
  for (int k = 0; k < N; ++k) {
    if ((double)S[k] > thresh) continue;
    const double sgn = signbit((double)Uw[(size_t)k * ld]) ? -1.0 : 1.0;  // Z15 flip recorded as -0.0
    for (;;) {
      for (int r = threadIdx.x; r < M; r += kCT) x[r] = (r == next_e) ? 1.0 : 0.0;
      ++next_e;
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
      if (res > 0.5 || next_e >= M) {
        for (int r = threadIdx.x; r < M; r += kCT) Uw[(size_t)k * ld + r] = (TI)(sgn * (x[r] / res));
        __syncthreads();
        break;
      }
    }
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
