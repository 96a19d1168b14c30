// common.cuh -- shared definitions of the CUDA path (kernels, planner, C-ABI). No oracle code.
#pragma once

#include <cstdint>
#include <cuda_runtime.h>

#include "wcsvd.h"

#define WCSVD_HD __host__ __device__ __forceinline__

namespace wcsvd {

constexpr double kU53 = 1.1102230246251565404e-16;  // 2^-53, fp64 unit roundoff

// ---------------------------------------------------------------------------------------------
// Round-robin (circle method) schedule, in "slot" form (§II.B; §IV.C).
// np slots hold the np indices; at every step the pairs are the fixed slot pairs (2k, 2k+1):
// top[k] = slot 2k, bot[k] = slot 2k+1. Between steps the contents move along one ring:
//   top[1] -> top[2] -> ... -> top[h-1] -> bot[h-1] -> bot[h-2] -> ... -> bot[0] -> top[1],
// with top[0] fixed (h = np/2). After np-1 steps every pair has met exactly once and every index
// is back in its own slot, so at sweep boundaries slot j holds original index j. Keeping pairs at
// fixed slots lets register-resident kernels use static register indices (the move is a rename).
// ---------------------------------------------------------------------------------------------
WCSVD_HD int rr_ring_index(int slot, int np) {  // position on the ring; -1 for the fixed slot 0
  const int h = np >> 1;
  if (slot == 0) return -1;
  const int k = slot >> 1;
  return (slot & 1) ? (2 * h - 2 - k) : (k - 1);
}
WCSVD_HD int rr_slot_of_ring(int r, int np) {
  const int h = np >> 1;
  return (r <= h - 2) ? 2 * (r + 1) : 2 * (2 * h - 2 - r) + 1;
}
// Slot a value in `slot` moves to after one step.
WCSVD_HD int rr_dest(int slot, int np) {
  if (slot == 0 || np == 2) return slot;
  const int L = np - 1;
  int r = rr_ring_index(slot, np) + 1;
  if (r == L) r = 0;
  return rr_slot_of_ring(r, np);
}
// Slot whose value moves into `slot` after one step (inverse of rr_dest).
WCSVD_HD int rr_src(int slot, int np) {
  if (slot == 0 || np == 2) return slot;
  const int L = np - 1;
  int r = rr_ring_index(slot, np) - 1;
  if (r < 0) r += L;
  return rr_slot_of_ring(r, np);
}
// Original index held by `slot` at step s (0 <= s < np-1).
WCSVD_HD int rr_content(int slot, int s, int np) {
  if (slot == 0 || np == 2) return slot;
  const int L = np - 1;
  int r = rr_ring_index(slot, np) - s;
  r %= L;
  if (r < 0) r += L;
  return rr_slot_of_ring(r, np);
}

// Per-matrix descriptor, built on the host by the planner and copied to the device.
struct MatDesc {
  const double* A;
  double* S;
  double* U;
  double* V;
  int* info;
  int* sweeps_inner;
  double* W;   // Level >= 1 working copy (m_pad x n_pad, ld m_pad), or nullptr
  double* Vw;  // Level >= 1 V accumulator (n_pad x n_pad, ld n_pad), or nullptr
  double tol;
  int m, n, lda, ldu, ldv;
  int M, N, swapped;
  int m_pad, n_pad, w, w2;
  int max_sweeps, inner_cap;
  int inner_cap2;  // W-cycle: cap on Level-2 sweeps per super-pair
  int withv;       // 1: accumulate V_x (requested as V, or as U when swapped); 0: values / U-only mode
  int fp32;        // 1: A, S, U, V hold float (wcsvd_batched_f32); the pointer fields are reinterpreted
  int idx;      // index of this matrix in the caller's batch (info / status arrays)
  int* status;  // internal per-matrix status flags (workspace), e.g. kNeedsCompletion
};

// Workspace slot pool: the Level-1 working copies (W + V) and the Level-0 two-phase park buffers are
// not allocated per matrix but per RESIDENT CTA (or cluster): a CTA takes a free slot when it starts
// (atomicCAS on busy[]) and returns it when it exits. nslots is the bucket's resident capacity; if more
// CTAs happen to be resident than slots exist, the extra ones wait -- never deadlocks, because slot
// holders wait on nothing the waiters hold. Which slot a matrix gets changes no arithmetic.
// The probe starts at the CTA's own SM's range (smid x per_sm): a slot there is held only by CTAs
// that ran on this SM, so with nslots = SMs x resident CTAs per SM a new CTA finds a free slot within
// per_sm probes (a start from blockIdx scanned ~nslots / 2 busy slots -- one global atomic round trip
// each -- and cost C2 ~45% of its time).
struct SlotPool {
  double* base;         // nslots x slot_doubles
  size_t slot_doubles;  // doubles per slot (the bucket's largest matrix)
  int* busy;            // [nslots], zero before the launch
  int nslots;
  int per_sm;           // slots per SM the pool was sized for (probe start = smid x per_sm)
};
__device__ __forceinline__ int slot_acquire(const SlotPool& p) {
  unsigned smid;
  asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
  const int start = (int)((smid * (unsigned)p.per_sm) % (unsigned)p.nslots);
  for (int i = start, tries = 0;; i = (i + 1 == p.nslots) ? 0 : i + 1) {
    if (atomicCAS(&p.busy[i], 0, 1) == 0) {
      __threadfence();
      return i;
    }
    if (++tries % p.nslots == 0) __nanosleep(256);  // every slot held: wait for an owner to finish
  }
}
__device__ __forceinline__ void slot_release(const SlotPool& p, int s) {
  __threadfence();
  atomicExch(&p.busy[s], 0);
}

// Status flags a kernel can leave for the completion pass (Z14): bit 0 = some sigma_j below the
// rank threshold; those U columns were written as 0 and need the deterministic MGS completion.
constexpr int kNeedsCompletion = 1;

}  // namespace wcsvd
