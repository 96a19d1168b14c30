// da.cu -- the data-assimilation consumer of the batched SVD (§V.F:
// "the data assimilation on each grid point involves one SVD. SVDs in different points can be batched
// together"; the paper's DA codes are ensemble Kalman filters, refs [36]-[38]).
//
// The paper does not write the analysis out; the reading (DESIGN.md §3 R-DA) is the ensemble-space
// analysis of the ensemble transform Kalman filter: with the scaled observation-space ensemble
// perturbations Y (m obs x n members) = U diag(S) V^T (economy SVD from wcsvd_batched) and the scaled
// innovation d (m), the analysis needs
//   T    = (I_n + Y^T Y)^(-1/2)            = I_n + V diag(g - 1) V^T,   g_i = (1 + s_i^2)^(-1/2)
//   wbar = (I_n + Y^T Y)^(-1) Y^T d          = V diag(s_i / (1 + s_i^2)) U^T d
// (the complement of span(V) has eigenvalue 1 of I + Y^T Y, so both forms hold for m < n too).
// One CTA per grid point: z = U^T d (warp dot products, fixed order), wbar = V (h .* z), and T by
// FP64 DMMA.8x8x4 tiles of (V diag(g - 1)) V^T plus the identity. Deterministic (no atomics).
#include <cuda_runtime.h>

#include "common.cuh"
#include "dmma.cuh"
#include "kernels.h"

namespace wcsvd {

namespace {
constexpr int kDaWarps = 8;
}

__global__ void __launch_bounds__(kDaWarps * 32) etkf_kernel(const DaDesc* __restrict__ descs) {
  const DaDesc q = descs[blockIdx.x];
  const int m = q.m, n = q.n, k = m < n ? m : n;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  extern __shared__ double sm[];
  double* s_z = sm;       // [k]  h_l (U^T d)_l
  double* s_g = sm + k;   // [k]  g_l - 1
  // z = U^T d, scaled by h = s / (1 + s^2); g - 1 with g = (1 + s^2)^(-1/2)
  for (int l = warp; l < k; l += kDaWarps) {
    const double* u = q.U + (size_t)l * m;
    double a = 0.0;
    for (int r = lane; r < m; r += 32) a = fma(u[r], q.d[r], a);
    for (int off = 16; off > 0; off >>= 1) a += __shfl_xor_sync(0xffffffffu, a, off);
    if (lane == 0) {
      const double s = q.S[l], p = fma(s, s, 1.0);
      s_z[l] = a * (s / p);
      s_g[l] = rsqrt(p) - 1.0;
    }
  }
  __syncthreads();
  // wbar = V (h .* z)
  for (int i = tid; i < n; i += kDaWarps * 32) {
    double a = 0.0;
    for (int l = 0; l < k; ++l) a = fma(q.V[(size_t)l * n + i], s_z[l], a);
    q.wbar[i] = a;
  }
  // T = I + (V diag(g - 1)) V^T: 8 x 8 output tiles per warp, k in steps of 4 (DMMA.8x8x4).
  // A fragment: A[r][c] = V[i0 + r][l + c] (g - 1)[l + c] at lane (r = lane/4, c = lane%4);
  // B fragment: B[c][j] = V[j0 + j][l + c] at lane (c = lane%4, j = lane/4).
  const int nt = (n + 7) / 8;
  for (int t = warp; t < nt * nt; t += kDaWarps) {
    const int i0 = (t % nt) * 8, j0 = (t / nt) * 8;
    const int ra = i0 + (lane >> 2), rb = j0 + (lane >> 2), c = lane & 3;
    double acc[2] = {0.0, 0.0};
    for (int l = 0; l < k; l += 4) {
      const int lc = l + c;
      const bool okc = lc < k;
      const double a = (okc && ra < n) ? q.V[(size_t)lc * n + ra] * s_g[lc] : 0.0;
      const double b = (okc && rb < n) ? q.V[(size_t)lc * n + rb] : 0.0;
      dmma884(acc, a, b);
    }
    const int row = i0 + (lane >> 2);
#pragma unroll
    for (int e = 0; e < 2; ++e) {
      const int col = j0 + 2 * (lane & 3) + e;
      if (row < n && col < n) q.T[(size_t)col * n + row] = acc[e] + (row == col ? 1.0 : 0.0);
    }
  }
}

cudaError_t launch_etkf(const DaDesc* descs, int count, int kmax, cudaStream_t stream) {
  if (count <= 0) return cudaSuccess;
  const size_t smem = sizeof(double) * 2 * (size_t)(kmax > 0 ? kmax : 1);
  etkf_kernel<<<count, kDaWarps * 32, smem, stream>>>(descs);
  return cudaGetLastError();
}

}  // namespace wcsvd
