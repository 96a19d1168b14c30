// dmma.cuh -- FP64 tensor-core tile primitives for sm_100a.
//
// B200 has no tcgen05 FP64 kind; its only FP64 MMA is DMMA.8x8x4 (warp-level mma.sync m8n8k4.f64),
// at the same 37 TF/s as DFMA (profiles/peaks_fp64_r01.json) but 8x fewer issue slots per flop.
// Fragment layouts (PTX ISA, mma.m8n8k4 .f64): lane l holds
//   A (8x4, row): A[l/4][l%4];  B (4x8, col): B[l%4][l/4];  C/D (8x8): C[l/4][2(l%4) + {0,1}].
#pragma once

namespace wcsvd {

__device__ __forceinline__ void dmma884(double (&c)[2], double a, double b) {
  asm("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};"
      : "+d"(c[0]), "+d"(c[1])
      : "d"(a), "d"(b));
}

}  // namespace wcsvd
