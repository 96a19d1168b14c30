// kernels.h -- launchers of the CUDA path (internal).
#pragma once
#include <cuda_runtime.h>

#include "common.cuh"

namespace wcsvd {

// Level-0 kernel variants (NP = padded columns, G column groups, R rows per thread).
enum L0Variant {
  kL0_8 = 1,    // NP=8,  G=1, R=8
  kL0_16 = 2,   // NP=16, G=2, R=8
  kL0_32 = 3,   // NP=32, G=2, R=4
  kL0_32s = 4,  // NP=32, G=2, R=1 (latency-bound small batches)
  kL0_48 = 5,   // NP=48, G=2, R=2
  kL0_64 = 6,   // NP=64, G=8, R=8
  kTP32 = 7,    // two-phase (l0_tp.cu): NP=32 (layouts: l0_tp.cu TPCfg)
  kTP64 = 8,    // two-phase (l0_tp.cu): NP=64
};
constexpr int kTP32MaxM = 128;  // planner limits of the two-phase variants (rows of the iterate)
constexpr int kTP64MaxM = 64;

// Level-1 Gram-path variants (pair panel width 2w, warps per CTA).
enum L1Variant {
  kL1_16x4 = 11,  // 2w = 16, 4 warps
  kL1_32x4 = 12,  // 2w = 32, 4 warps
  kL1_32x8 = 13,  // 2w = 32, 8 warps
};

// Level-1 launch: `cluster` CTAs per matrix (1, 2, 4 or 8; a thread-block cluster when > 1).
// wcycle = 1: the W-cycle kernel (Level 1 -> Level 2 recursion, one CTA per matrix); 2: the group (i)
// PANEL path (one-sided Jacobi of the CholeskyQR-compressed pair panel, 2w = 32, fp64 working copy).
// fp32 = 1: float I/O; f32_compute = 1 iterates in fp32 (FFMA), else on an fp64 working copy (DMMA).
cudaError_t launch_l1(int variant, int wcycle, int fp32, int f32_compute, const MatDesc* descs, const int* order,
                      int count, int cluster, const SlotPool& pool, cudaStream_t stream);

cudaError_t launch_l0tp(int variant, int fp32, const MatDesc* descs, const int* order, int count, int maxM,
                        const SlotPool& pool, cudaStream_t stream);
size_t l0tp_park_bytes(int variant, int M);  // per-matrix park buffer (X and V_x registers), fp64
int l0tp_occupancy(int variant, int fp32, int maxM);  // resident CTAs per SM (-1 if unknown)

cudaError_t launch_l0(int variant, int withv, int fp32, const MatDesc* descs, const int* order, int count,
                      int maxM, cudaStream_t stream);

}  // namespace wcsvd

namespace wcsvd {
cudaError_t launch_complete(int fp32, const MatDesc* descs, int count, cudaStream_t stream);
}  // namespace wcsvd

namespace wcsvd {
// Data-assimilation consumer (da.cu): per grid point, the ETKF ensemble-space analysis from an SVD.
struct DaDesc {
  const double* S;  // k = min(m, n)
  const double* U;  // m x k, ld m
  const double* V;  // n x k, ld n
  const double* d;  // m
  double* wbar;     // n
  double* T;        // n x n, ld n
  int m, n;
};
cudaError_t launch_etkf(const DaDesc* descs, int count, int kmax, cudaStream_t stream);
}  // namespace wcsvd
