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
};

// Level-1 Gram-path variants (pair panel width 2w, warps per CTA).
enum L1Variant {
  kL1_16x4 = 11,  // 2w = 16, 4 warps
  kL1_32x4 = 12,  // 2w = 32, 4 warps
  kL1_32x8 = 13,  // 2w = 32, 8 warps
};

cudaError_t launch_l1(int variant, int fp32, const MatDesc* descs, const int* order, int count, cudaStream_t stream);

cudaError_t launch_l0(int variant, int withv, int fp32, const MatDesc* descs, const int* order, int count,
                      int maxM, cudaStream_t stream);

}  // namespace wcsvd

namespace wcsvd {
cudaError_t launch_complete(int fp32, const MatDesc* descs, int count, cudaStream_t stream);
}  // namespace wcsvd
