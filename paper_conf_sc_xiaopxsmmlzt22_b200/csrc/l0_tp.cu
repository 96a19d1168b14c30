// l0_tp.cu -- Level-0 batched SVD kernel, "two-phase" form: the whole one-sided Jacobi of a matrix
// that fits on-chip in one CTA (Alg 2 l.2-3; Step 1; §IV.B,
// PAPER.md:232-243), with the X iteration and the V accumulation time-multiplexed through the same
// registers.
//
// Why. In one-sided Jacobi only X = A V couples the rows (the dot products
// gamma_k of every step need all rows of X); the rows of V never interact: V <- V G_1 G_2 ... is a
// row-by-row replay of the rotation sequence that X produced (eq 2). The fused
// kernel (l0_jacobi.cu) keeps X and V in registers side by side, so a 64 x 64 matrix needs
// 2 x 4096 doubles of registers and only two matrices fit an SM -- too few warps to hide the
// latency of the per-step reduction -> rotation -> update chain. Here the CTA runs one sweep of
// X (storing the sweep's rotations (c, s) in shared memory), parks X in global memory (L2), loads
// V, replays the sweep's rotations on V at full FMA rate (no reduction, no barrier), parks V and
// reloads X. Registers hold one matrix at a time, so twice as many matrices are resident per SM,
// and the X phase of one CTA overlaps the barrier-free V phase of another.
//
// X phase (per step, PAPER.md:64 round-robin in slot form, common.cuh): (1) every row-thread forms
// its partial gamma_k over its R rows (and alpha, beta at the first step of a sweep);
// barrier; (2) warp 0 alone (lane k = pair k) sums the partials in a fixed order, evaluates eq (4)
// (rotation.cuh, R-ROT), stores (c_k, s_k) and updates the cached norms by eq (6) in its closed
// form; barrier; (3) every thread rotates its rows (eq 3) and moves the slots along the ring.
// V phase: step (3) only, on the rows of V, reading the stored (c, s). The same (c, s) bits and the
// same update formula are applied to X and to V, so V is exactly the product the fused kernel
// would have accumulated. A sweep that applies no rotation ends the iteration (Z6) and is not
// replayed (its rotations are all (1, 0) and its slot moves form a full cycle: the identity).
#include <cuda_runtime.h>

#include <cmath>

#include "common.cuh"
#include "kernels.h"
#include "prec.cuh"
#include "rotation.cuh"

namespace wcsvd {

namespace {

#ifdef WCSVD_PHASE_PROFILE
// Debug builds only (-DWCSVD_PHASE_PROFILE): clock64() totals of lane 0 of every warp:
// [0] phase 1 + first barrier, [1] serial section (+ second barrier), [2] rotate + move,
// [3] V phase, [4] park / unpark, [5] X steps, [6] V sweeps.
__device__ unsigned long long g_tp_cycles[8];
#define TP_T(v) long long v = clock64()
#define TP_ADD(i, dt) \
  do { if ((threadIdx.x & 31) == 0) atomicAdd(&g_tp_cycles[i], (unsigned long long)(dt)); } while (0)
#else
#define TP_T(v) (void)0
#define TP_ADD(i, dt) (void)0
#endif

// Rotate this thread's R rows x NL slot-columns (local pair j = slots (2j, 2j+1), (c, s) = cs[j];
// eq (3)) and move every slot one step along the circle-method ring (common.cuh):
// outputs of local pair j go top -> top[j+1], bot -> bot[j-1]; group 0 keeps top[0] and sends
// bot[0] to its top[1]; other groups receive top[0] from the left neighbour lane; the last group
// moves its last top to its last bot, the others receive their last bot from the right.
// The (c, s) of local pair j sit at cs[(j / SUB) (SUB + 1) + j % SUB] (runs of SUB pairs, padded
// by one entry against shared-memory bank conflicts).
template <typename T, int NP, int G, int R, int SUB>
__device__ __forceinline__ void rotate_move(const T (&x)[R][NP / G], T (&y)[R][NP / G],
                                            const typename Prec<T>::V2* __restrict__ cs, int g) {
  using V2 = typename Prec<T>::V2;
  constexpr int NL = NP / G;
  constexpr int LP = NL / 2;
  T top0[R], send_l[R], send_r[R];
#pragma unroll
  for (int j = 0; j < LP; ++j) {
    const V2 p = cs[(j / SUB) * (SUB + 1) + (j % SUB)];
#pragma unroll
    for (int r = 0; r < R; ++r) {
      const T a = x[r][2 * j], b = x[r][2 * j + 1];
      const T na = fma(p.y, b, p.x * a);
      const T nb = fma(-p.y, a, p.x * b);
      if (j == 0) top0[r] = na;
      else if (j + 1 < LP) y[r][2 * (j + 1)] = na;
      else send_r[r] = na;
      if (j == 0) send_l[r] = nb;
      else y[r][2 * (j - 1) + 1] = nb;
    }
  }
  const bool gfirst = (g == 0), glast = (g == G - 1);
#pragma unroll
  for (int r = 0; r < R; ++r) {
    T from_left = 0, from_right = 0;
    if (G > 1) {
      from_left = __shfl_up_sync(0xffffffffu, send_r[r], 1);
      from_right = __shfl_down_sync(0xffffffffu, send_l[r], 1);
    }
    y[r][0] = gfirst ? top0[r] : from_left;
    y[r][2] = gfirst ? send_l[r] : top0[r];
    y[r][2 * (LP - 1) + 1] = glast ? send_r[r] : from_right;
  }
}

template <typename T>
struct TPCtx {
  using V2 = typename Prec<T>::V2;
  T* part;       // [parity (RED only)][3][RW4][PS] partial gamma / alpha / beta per (row-thread, pair)
  T* nrm;        // [2 parity][NP] cached squared norms per slot (RED: this warp's copy)
  V2* csw;       // RED: this warp's [GX][LPX+1] (c, s) of the current step
  V2* rot;       // [NP-1][GX][LPX+1] (c, s) of every step of the current sweep
  int RW4, PS;
  int lane, warp, g, rt;
  bool isW;
  int dtop, dbot;  // warp 0, lane k: the slots that the contents of slots 2k, 2k+1 move to
  T tol2;
  int par;         // step parity (norm cache double buffer)
  int nwarp;       // warps per CTA; the rotations of step s are evaluated by warp s % nwarp
  int* rot_flag;   // set to 1 when some pair of the current sweep rotates
#ifdef WCSVD_PHASE_PROFILE
  long long acc[3];
#endif
};

// One X step: partial dot products -> barrier -> the step's rotations (fixed-order sums, eq (4),
// eq (6)) -> rotate and move (the rotations of `step` are kept for the V phase). RED = false: one
// warp evaluates the rotations (warp s % nwarp, spreading the serial part over the sub-partitions)
// and a second barrier publishes them. RED = true: every warp evaluates all of them (bitwise the
// same numbers), so one barrier per step suffices; the partials are double-buffered by parity.
template <typename T, int NP, int G, int R, bool FIRST, bool RED, int RWM>
__device__ __forceinline__ void x_step(TPCtx<T>& cx, const T (&x)[R][NP / G], T (&y)[R][NP / G], int step) {
  constexpr int NL = NP / G;
  constexpr int LP = NL / 2;
  constexpr int NPAIR = NP / 2;
  const int SEC = cx.RW4 * cx.PS;
  T* part = cx.part + (RED ? cx.par * 3 * SEC : 0);
  TP_T(t0);
  {
    // rows outer, pairs inner: LP independent accumulation chains interleave (each still sums its
    // rows in order 0 .. R-1); rows >= M (row-threads past RW) contribute zeros
    T gm[LP], al[LP], be[LP];
#pragma unroll
    for (int j = 0; j < LP; ++j) gm[j] = al[j] = be[j] = 0;
    if (cx.isW) {
#pragma unroll
      for (int r = 0; r < R; ++r) {
#pragma unroll
        for (int j = 0; j < LP; ++j) {
          gm[j] = fma(x[r][2 * j], x[r][2 * j + 1], gm[j]);
          if (FIRST) {
            al[j] = fma(x[r][2 * j], x[r][2 * j], al[j]);
            be[j] = fma(x[r][2 * j + 1], x[r][2 * j + 1], be[j]);
          }
        }
      }
    }
    if constexpr (!RED) {
      // one-warp rotation evaluation: the 32 / G row-threads of a warp pre-sum their partials by a
      // fixed xor tree (the same bits in every lane of a group), so the serial warp adds one partial
      // per warp instead of one per row-thread
#pragma unroll
      for (int o = G; o < 32; o <<= 1)
#pragma unroll
        for (int j = 0; j < LP; ++j) {
          gm[j] += __shfl_xor_sync(0xffffffffu, gm[j], o);
          if (FIRST) {
            al[j] += __shfl_xor_sync(0xffffffffu, al[j], o);
            be[j] += __shfl_xor_sync(0xffffffffu, be[j], o);
          }
        }
      if (cx.lane < G) {
        const int base = cx.warp * cx.PS + cx.g * LP;
#pragma unroll
        for (int j = 0; j < LP; ++j) {
          part[base + j] = gm[j];
          if (FIRST) {
            part[SEC + base + j] = al[j];
            part[2 * SEC + base + j] = be[j];
          }
        }
      }
    } else if (cx.isW) {
      const int base = cx.rt * cx.PS + cx.g * LP;
#pragma unroll
      for (int j = 0; j < LP; ++j) {
        part[base + j] = gm[j];
        if (FIRST) {
          part[SEC + base + j] = al[j];
          part[2 * SEC + base + j] = be[j];
        }
      }
    }
  }
  __syncthreads();
  TP_T(t1);
  // Stored rotations: padded [GX][LP+1] per step when warps read them back here (bank
  // conflicts), packed [NPAIR] when only the V phase reads them (RED: all lanes broadcast).
  constexpr int RSTEP = RED ? NPAIR : G * (LP + 1);
  typename Prec<T>::V2* rs = cx.rot + step * RSTEP;
  if (RED || cx.warp == step % cx.nwarp) {
    const int k = cx.lane;
    bool rot = false;
    if (k < NPAIR) {
      const int PS = cx.PS;
      T g4[4] = {0, 0, 0, 0}, a4[4] = {0, 0, 0, 0}, b4[4] = {0, 0, 0, 0};
      // RWM (compile time) >= RW4: fully unrolled, so the loads of a block issue back to back
#pragma unroll
      for (int i = 0; i < RWM; i += 4) {  // rows [RW, RW4) are zero
        if (i >= (RED ? cx.RW4 : cx.nwarp)) break;  // !RED: one pre-summed partial per warp
#pragma unroll
        for (int u = 0; u < 4; ++u) {
          g4[u] += part[(i + u) * PS + k];
          if (FIRST) {
            a4[u] += part[SEC + (i + u) * PS + k];
            b4[u] += part[2 * SEC + (i + u) * PS + k];
          }
        }
      }
      const T gm = (g4[0] + g4[1]) + (g4[2] + g4[3]);
      T al, be;
      if (FIRST) {
        al = (a4[0] + a4[1]) + (a4[2] + a4[3]);
        be = (b4[0] + b4[1]) + (b4[2] + b4[3]);
      } else {
        al = cx.nrm[cx.par * NP + 2 * k];
        be = cx.nrm[cx.par * NP + 2 * k + 1];
      }
      T c, sn, t;
      rot = jacobi_rotation(al, be, gm, cx.tol2, c, sn, t);
      const int o = (k / LP) * (LP + 1) + (k % LP);
      if (!RED) rs[o] = Prec<T>::mk(c, sn);
      if (RED && cx.warp == 0) rs[k] = Prec<T>::mk(c, sn);
      if (RED) cx.csw[o] = Prec<T>::mk(c, sn);
      // eq (6) in closed form: alpha' = alpha + t gamma, beta' = beta - t gamma
      cx.nrm[(cx.par ^ 1) * NP + cx.dtop] = rot ? fma(t, gm, al) : al;
      cx.nrm[(cx.par ^ 1) * NP + cx.dbot] = rot ? fma(-t, gm, be) : be;
    }
    if (__ballot_sync(0xffffffffu, rot) != 0u && k == 0 && (!RED || cx.warp == 0)) *cx.rot_flag = 1;
  }
  if (RED) __syncwarp();
  else __syncthreads();
  TP_T(t2);
  rotate_move<T, NP, G, R, LP>(x, y, (RED ? cx.csw : rs) + cx.g * (LP + 1), cx.g);
  cx.par ^= 1;
#ifdef WCSVD_PHASE_PROFILE
  TP_T(t3);
  cx.acc[0] += t1 - t0;
  cx.acc[1] += t2 - t1;
  cx.acc[2] += t3 - t2;
#endif
}

// One sweep of NP-1 (odd) steps from a; ends in b with every slot back in its original column.
template <typename T, int NP, int G, int R, bool RED, int RWM>
__device__ __forceinline__ void x_sweep(TPCtx<T>& cx, T (&a)[R][NP / G], T (&b)[R][NP / G]) {
  x_step<T, NP, G, R, true, RED, RWM>(cx, a, b, 0);
#pragma unroll 1
  for (int s = 1; s < NP - 1; s += 2) {
    x_step<T, NP, G, R, false, RED, RWM>(cx, b, a, s);
    x_step<T, NP, G, R, false, RED, RWM>(cx, a, b, s + 1);
  }
}

// V phase: replay the sweep's stored rotations on this thread's row of V (R = 1 row, NP/GV slots).
// `rot` + the group offset of this thread; the stored layout is the X phase's [GX][LPX+1] per step.
// PACKED: the rotations are stored as [NPAIR] per step, else as the X phase's padded [GX][LPX+1].
template <typename T, int NP, int GV, int GX, bool PACKED>
__device__ __forceinline__ void v_sweep(const typename Prec<T>::V2* __restrict__ rot, int gv, T (&a)[1][NP / GV],
                                        T (&b)[1][NP / GV]) {
  constexpr int LPX = NP / GX / 2;
  constexpr int LPV = NP / GV / 2;
  constexpr int STEP = PACKED ? NP / 2 : GX * (LPX + 1);
  constexpr int SUB = PACKED ? NP / 2 : LPX;
  // local pair j of group gv is global pair k = gv LPV + j, stored at (k / SUB)(SUB + 1) + k % SUB;
  // LPV is a multiple of LPX (GV <= GX), so group gv's pairs are LPV / LPX padded runs of LPX.
  static_assert(PACKED || LPV % LPX == 0, "V groups must be unions of X groups");
  const typename Prec<T>::V2* cs = rot + (PACKED ? gv * LPV : gv * (LPV / LPX) * (LPX + 1));
  rotate_move<T, NP, GV, 1, SUB>(a, b, cs, gv);
#pragma unroll 1
  for (int s = 1; s < NP - 1; s += 2) {
    rotate_move<T, NP, GV, 1, SUB>(b, a, cs + s * STEP, gv);
    rotate_move<T, NP, GV, 1, SUB>(a, b, cs + (s + 1) * STEP, gv);
  }
}

// Park stores with an L2 evict_last priority (build option WCSVD_TP_PARK_HINT=1): the slot is read back
// one phase later by the same CTA, while A, U, V and S stream through L2 once (evict-first loads /
// stores). Measured on C2: DRAM writes 1.50 -> 0.84 GB per launch (total 1.18 GB = 1.19x the 0.99 GB
// compulsory, from 1.83 GB) but 18.05 / 18.51 vs 17.77 / 17.79 ms, so the default stays plain.
#ifndef WCSVD_TP_PARK_HINT
#define WCSVD_TP_PARK_HINT 0
#endif
__device__ __forceinline__ void st_last(double* p, double v, unsigned long long pol) {
  asm volatile("st.global.L2::cache_hint.f64 [%0], %1, %2;" ::"l"(p), "d"(v), "l"(pol) : "memory");
}
__device__ __forceinline__ void st_last(float* p, float v, unsigned long long pol) {
  asm volatile("st.global.L2::cache_hint.f32 [%0], %1, %2;" ::"l"(p), "f"(v), "l"(pol) : "memory");
}
template <typename T, int R, int NL>
__device__ __forceinline__ void park(T* __restrict__ buf, const T (&x)[R][NL], int tid, int nt) {
#if WCSVD_TP_PARK_HINT
  unsigned long long pol;
  asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(pol));
#endif
#pragma unroll
  for (int r = 0; r < R; ++r)
#pragma unroll
    for (int l = 0; l < NL; ++l) {
#if WCSVD_TP_PARK_HINT
      st_last(buf + (size_t)(r * NL + l) * nt + tid, x[r][l], pol);
#else
      __stcg(buf + (size_t)(r * NL + l) * nt + tid, x[r][l]);
#endif
    }
}
template <typename T, int R, int NL>
__device__ __forceinline__ void unpark(const T* __restrict__ buf, T (&x)[R][NL], int tid, int nt) {
#pragma unroll
  for (int r = 0; r < R; ++r)
#pragma unroll
    for (int l = 0; l < NL; ++l) x[r][l] = __ldcg(buf + (size_t)(r * NL + l) * nt + tid);
}

}  // namespace

// Elements (of T) of the region that holds the sweep's rotations and, at finalisation, the
// [RW4][NP] sign-rule scratch.
template <int NP, int GX, bool RED>
__host__ __device__ constexpr int rot_region(int RW4) {
  return 2 * (NP - 1) * (RED ? NP / 2 : GX * (NP / GX / 2 + 1)) > RW4 * NP
             ? 2 * (NP - 1) * (RED ? NP / 2 : GX * (NP / GX / 2 + 1))
             : RW4 * NP;
}

// Shared-memory bytes of one CTA (must match the carve-up in the kernel).
template <typename T, int NP, int GX, int RX, bool RED>
size_t l0tp_smem_bytes(int M, int threads) {
  constexpr int LPX = NP / GX / 2;
  const int RW4 = ((M + RX - 1) / RX + 3) / 4 * 4;  // the warp-local hand-off (2 GX 16 RX) fits 3 RW4 PS for RW4 = 16
  const int PS = NP / 2 + 1;
  const int NCOPY = RED ? threads / 32 : 1;  // norm caches (and cs buffers) per CTA
  return 16 + sizeof(T) * (RED ? 6 : 3) * (size_t)RW4 * PS + sizeof(T) * 2 * NP * NCOPY
         + (RED ? 2 * sizeof(T) * (size_t)NCOPY * GX * (LPX + 1) : 0)
         + sizeof(T) * rot_region<NP, GX, RED>(RW4)
         + sizeof(T) * 2 * NP + sizeof(int) * (NP + 8);
}

// Park-buffer elements per matrix (X phase registers + V phase registers of every thread).
template <int NP, int GX, int RX, int GV>
constexpr size_t l0tp_park_elems(int nt) {
  return (size_t)nt * (RX * (NP / GX) + NP / GV);
}

// One CTA per matrix. X phase: thread t = (row-thread rt = t / GX, group g = t % GX) holds rows
// rt*RX .. rt*RX+RX-1 x slots g*NP/GX .. of X. V phase: thread t = (row rv = t / GV, group
// gv = t % GV) holds row rv x slots gv*NP/GV .. of V_x.
template <typename T, int NP, int GX, int RX, int GV, bool RED, int MAXT, int MINB>
__global__ void __launch_bounds__(MAXT, MINB) l0tp_kernel(const MatDesc* __restrict__ descs,
                                                          const int* __restrict__ order, SlotPool pool) {
  using V2 = typename Prec<T>::V2;
  constexpr int NLX = NP / GX;
  constexpr int LPX = NLX / 2;
  constexpr int NPAIR = NP / 2;
  constexpr int NLV = NP / GV;
  const MatDesc d = descs[order[blockIdx.x]];
  const int M = d.M, N = d.N;
  const int RW = (M + RX - 1) / RX;
  const int RW4 = (RW + 3) / 4 * 4;
  const int PS = NPAIR + 1;
  const int NT = blockDim.x;
  const int tid = threadIdx.x;
  const int lane = tid & 31, warp = tid >> 5;
  // X-phase layout: row-thread rt = t / GX, group g = t % GX
  const int g = tid % GX, rt = tid / GX;
  const bool isW = rt < RW;
  const int gv = tid % GV, rv = tid / GV;
  const bool withv = d.withv != 0;

  extern __shared__ __align__(16) unsigned char smem_raw[];
  unsigned long long* s_max = reinterpret_cast<unsigned long long*>(smem_raw);  // 16 B
  const int NCOPY = RED ? NT / 32 : 1;
  T* s_part = reinterpret_cast<T*>(smem_raw + 16);                        // [RED ? 2 : 1][3][RW4][PS]
  T* s_nrm = s_part + (RED ? 6 : 3) * RW4 * PS;                           // [NCOPY][2][NP]
  V2* s_csw = reinterpret_cast<V2*>(s_nrm + NCOPY * 2 * NP);              // RED: [NCOPY][GX][LPX+1]
  V2* s_rot = s_csw + (RED ? NCOPY * GX * (LPX + 1) : 0);                 // [NP-1][GX][LPX+1]
  T* s_sig = reinterpret_cast<T*>(s_rot) + rot_region<NP, GX, RED>(RW4);  // [NP]
  T* s_sgn = s_sig + NP;                                                  // [NP]
  int* s_rank = reinterpret_cast<int*>(s_sgn + NP);                       // [NP]
  int* s_flags = s_rank + NP;                                             // [8]
  T* s_vbest = reinterpret_cast<T*>(s_rot);  // finalisation: [RW4][NP] sign-rule scratch (aliases s_rot)
  __shared__ int s_slot;  // park-buffer slot of this CTA (SlotPool: sized to resident CTAs, not the batch)
  if (tid < 8) s_flags[tid] = 0;
  if (tid == 0) {
    *s_max = 0ull;
    s_slot = slot_acquire(pool);
  }
  for (int e = tid; e < (RED ? 6 : 3) * RW4 * PS; e += NT) s_part[e] = T(0);
  __syncthreads();

  // ---- Stage-in: X = A (m >= n) or A^T (m < n), zero-padded. ----
  T xa[RX][NLX], xb[RX][NLX];
  bool bad = false;
  T amax = 0;
  const T* Ain = reinterpret_cast<const T*>(d.A);
#pragma unroll
  for (int r = 0; r < RX; ++r) {
#pragma unroll
    for (int l = 0; l < NLX; ++l) {
      const int col = g * NLX + l;
      const int row = rt * RX + r;
      T v = 0;
      if (isW && row < M && col < N) {
        // A is read once: streaming loads (evict-first), so the park slots keep their place in L2
        v = __ldcs(d.swapped ? Ain + (size_t)row * d.lda + col : Ain + (size_t)col * d.lda + row);
        bad |= !isfinite(v);
        amax = fmax(amax, fabs(v));
      }
      xa[r][l] = v;
    }
  }
  if (bad) atomicOr(&s_flags[2], 1);
  if (isW && amax > T(0)) atomicMax(s_max, (unsigned long long)__double_as_longlong((double)amax));
  __syncthreads();
  const bool nonfinite = s_flags[2] != 0;
  // Exact power-of-two pre-scaling to max|x| in [0.5, 1) (see l0_jacobi.cu).
  int sexp = 0;
  if (!nonfinite && *s_max != 0ull) {
    frexp(__longlong_as_double((long long)*s_max), &sexp);
    const T f = (T)ldexp(1.0, -sexp);
#pragma unroll
    for (int r = 0; r < RX; ++r)
#pragma unroll
      for (int l = 0; l < NLX; ++l) xa[r][l] *= f;
  }

  TPCtx<T> cx;
#ifdef WCSVD_PHASE_PROFILE
  cx.acc[0] = cx.acc[1] = cx.acc[2] = 0;
#endif
  cx.part = s_part;
  cx.nrm = s_nrm + (RED ? warp * 2 * NP : 0);
  cx.csw = s_csw + (RED ? warp * GX * (LPX + 1) : 0);
  cx.rot = s_rot;
  cx.RW4 = RW4;
  cx.PS = PS;
  cx.lane = lane;
  cx.warp = warp;
  cx.g = g;
  cx.rt = rt;
  cx.isW = isW;
  cx.dtop = rr_dest(2 * lane, NP);
  cx.dbot = rr_dest(2 * lane + 1, NP);
  cx.tol2 = (T)(d.tol * d.tol);
  cx.par = 0;
  cx.nwarp = NT / 32;
  T* parkX = reinterpret_cast<T*>(pool.base + (size_t)s_slot * pool.slot_doubles);
  T* parkV = parkX + (size_t)NT * RX * NLX;
  int sweep = 0;
  bool converged = false;
  bool vmat = false;  // V_x materialised in parkV (else V_x = I)
  if (!nonfinite) {
    for (;;) {
      cx.rot_flag = &s_flags[4 + (sweep & 1)];
      // this sweep's flag was cleared one sweep earlier (or at start); clear the next one (its last
      // readers passed the barrier that ended the previous loop iteration)
      if (tid == 0) s_flags[4 + ((sweep + 1) & 1)] = 0;
      x_sweep<T, NP, GX, RX, RED, (MAXT / GX + 3) / 4 * 4>(cx, xa, xb);  // ends in xb, slots in order
      ++sweep;
      __syncthreads();
      const bool any = *cx.rot_flag != 0;
      if (any && withv) {
        // park X, replay this sweep's rotations on V_x, park V_x, reload X
        TP_T(p0);
        park<T, RX, NLX>(parkX, xb, tid, NT);
        T va[1][NLV], vb[1][NLV];
        if (vmat) {
          unpark<T, 1, NLV>(parkV, va, tid, NT);
        } else {
#pragma unroll
          for (int l = 0; l < NLV; ++l) va[0][l] = (rv == gv * NLV + l) ? T(1) : T(0);
        }
        TP_T(p1);
        v_sweep<T, NP, GV, GX, RED>(s_rot, gv, va, vb);
        TP_T(p2);
        park<T, 1, NLV>(parkV, vb, tid, NT);
        vmat = true;
        unpark<T, RX, NLX>(parkX, xa, tid, NT);
#ifdef WCSVD_PHASE_PROFILE
        // consume the loads before reading the clock
        if (xa[0][0] == T(12345.678)) s_flags[7] = 1;
        TP_T(p3);
        TP_ADD(3, p2 - p1);
        TP_ADD(4, (p1 - p0) + (p3 - p2));
        TP_ADD(6, 1);
#endif
      } else {
#pragma unroll
        for (int r = 0; r < RX; ++r)
#pragma unroll
          for (int l = 0; l < NLX; ++l) xa[r][l] = xb[r][l];
      }
      if (!any) { converged = true; break; }
      if (sweep >= d.max_sweeps) break;
      __syncthreads();  // the next sweep overwrites s_rot and clears the other rotation flag
    }
  }

#ifdef WCSVD_PHASE_PROFILE
  TP_ADD(0, cx.acc[0]);
  TP_ADD(1, cx.acc[1]);
  TP_ADD(2, cx.acc[2]);
  TP_ADD(5, sweep * (NP - 1));
#endif
  // ---- Finalisation: sigma_j = ||x_j|| (fresh, fixed order), stable descending
  // rank (Z15), U = X / sigma, sign rule on the square factor V_x (Z15), un-orientation.
  __syncthreads();
  if (isW) {
#pragma unroll
    for (int l = 0; l < NLX; ++l) {
      T a = 0;
#pragma unroll
      for (int r = 0; r < RX; ++r) a = fma(xa[r][l], xa[r][l], a);
      const int col = g * NLX + l;  // [RW][NP] view over the first two partial sections
      s_part[(col < NPAIR ? 0 : RW4) * PS + rt * PS + (col % NPAIR)] = a;
    }
  }
  // Without V_x (values / U-only mode) the sign rule is applied to the columns of X.
  if (!withv && isW) {
#pragma unroll
    for (int l = 0; l < NLX; ++l) {
      T best = 0;
#pragma unroll
      for (int r = 0; r < RX; ++r)
        if (fabs(xa[r][l]) > fabs(best)) best = xa[r][l];
      s_vbest[rt * NP + g * NLX + l] = best;
    }
  }
  __syncthreads();
  for (int j = tid; j < NP; j += NT) {
    const int base = (j < NPAIR ? 0 : RW4) * PS + (j % NPAIR);
    T a4[4] = {0, 0, 0, 0};
    for (int i = 0; i < RW; i += 4) {
#pragma unroll
      for (int u = 0; u < 4; ++u) a4[u] += s_part[base + (i + u) * PS];
    }
    s_sig[j] = sqrt((a4[0] + a4[1]) + (a4[2] + a4[3]));  // of the pre-scaled X
    T best = 0;
    if (!withv) {
      for (int i = 0; i < RW; ++i) {
        const T v = s_vbest[i * NP + j];
        if (fabs(v) > fabs(best)) best = v;
      }
    } else if (!vmat) {
      best = T(1);  // V_x = I
    } else if (j < N) {
      // largest-|.| entry of column j of V_x (first on ties): rows in increasing order
      const T* col = parkV + (size_t)(j % NLV) * NT + j / NLV;
      for (int r = 0; r < N; ++r) {
        const T v = __ldcg(col + r * GV);
        if (fabs(v) > fabs(best)) best = v;
      }
    }
    s_sgn[j] = (best < T(0)) ? T(-1) : T(1);
  }
  __syncthreads();
  for (int j = tid; j < NP; j += NT) {
    int rk = -1;
    if (j < N && nonfinite) {
      rk = j;  // NaN sigmas: identity order, every column written
    } else if (j < N) {
      rk = 0;
      const T sj = s_sig[j];
      for (int i = 0; i < N; ++i) {
        const T si = s_sig[i];
        rk += (si > sj) || (si == sj && i < j);
      }
    }
    s_rank[j] = rk;
  }
  __syncthreads();
  T sig1 = 0;
  for (int i = 0; i < N; ++i) sig1 = fmax(sig1, s_sig[i]);
  const T thresh = sig1 * (T)M * Prec<T>::eps;  // Z14 rank threshold (scale-invariant)
  const T nanv = Prec<T>::qnan();
  // X-space factors: U_w -> U (V if swapped), V_x -> V (U if swapped).
  T* dstW = reinterpret_cast<T*>(d.swapped ? d.V : d.U);
  const int ldW = d.swapped ? d.ldv : d.ldu;
  T* dstV = reinterpret_cast<T*>(d.swapped ? d.U : d.V);
  const int ldV = d.swapped ? d.ldu : d.ldv;
  bool needs_completion = false;
  if (isW && dstW) {
#pragma unroll
    for (int l = 0; l < NLX; ++l) {
      const int col = g * NLX + l;
      if (col < N) {
        const int rk = s_rank[col];
        const T sj = s_sig[col];
        const T sgn = s_sgn[col];
        const bool ok = sj > thresh;
        needs_completion |= !ok;
#pragma unroll
        for (int r = 0; r < RX; ++r) {
          const int row = rt * RX + r;
          if (row < M)  // rank-deficient columns: signed zero, completed by complete_u_kernel
            __stcs(dstW + (size_t)rk * ldW + row, nonfinite ? nanv : (ok ? sgn * (xa[r][l] / sj) : sgn * T(0)));
        }
      }
    }
  }
  if (withv && dstV) {
    for (int e = tid; e < N * N; e += NT) {
      const int r = e % N, c = e / N;
      T v = (r == c) ? T(1) : T(0);
      if (vmat) v = __ldcs(parkV + (size_t)(c % NLV) * NT + r * GV + c / NLV);  // last read of the slot
      __stcs(dstV + (size_t)s_rank[c] * ldV + r, nonfinite ? nanv : s_sgn[c] * v);
    }
  }
  if (needs_completion && !nonfinite) atomicOr(&s_flags[3], 1);
  T* Sout = reinterpret_cast<T*>(d.S);
  for (int j = tid; j < N; j += NT) __stcs(Sout + s_rank[j], nonfinite ? nanv : (T)ldexp((double)s_sig[j], sexp));
  __syncthreads();
  if (tid == 0) {
    if (d.info) d.info[d.idx] = nonfinite ? -2 : (converged ? sweep : -1);
    if (d.sweeps_inner) d.sweeps_inner[d.idx] = 0;
    if (d.status) d.status[d.idx] = (s_flags[3] && dstW) ? kNeedsCompletion : 0;
    slot_release(pool, s_slot);
  }
}

// ---- launcher ----
// Threads of a CTA: enough for the X-phase row-threads and the V-phase rows.
template <int NP, int GX, int RX, int GV>
constexpr int tp_threads(int M) {
  return (((M + RX - 1) / RX * GX > NP * GV ? (M + RX - 1) / RX * GX : NP * GV) + 31) / 32 * 32;
}

template <typename T, int NP, int GX, int RX, int GV, bool RED, int MAXT, int MINB>
static cudaError_t launch_tp_t(const MatDesc* descs, const int* order, int count, int maxM, const SlotPool& pool,
                               cudaStream_t stream) {
  const int threads = tp_threads<NP, GX, RX, GV>(maxM);
  if (threads > MAXT) return cudaErrorInvalidConfiguration;
  const size_t smem = l0tp_smem_bytes<T, NP, GX, RX, RED>(maxM, threads);
  auto kern = l0tp_kernel<T, NP, GX, RX, GV, RED, MAXT, MINB>;
  cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  kern<<<count, threads, smem, stream>>>(descs, order, pool);
  return cudaGetLastError();
}

// Variant configurations: X layout (GX groups, RX rows per thread), V layout (GV groups, one row
// per thread), rotation evaluation (RED: every warp, else one warp), launch bounds. The planner's M
// limits (kernels.h) bound the thread count of every bucket.
// Variant configurations: X layout (GX groups, RX rows per thread), V layout (GV groups, one row
// per thread), rotation evaluation (RED: every warp, else one warp), launch bounds. Measured
// alternatives for NP = 64 (r01): every warp reduces (RED, 128 threads) 24.4 ms,
// 8 rows per thread with 64 threads 21.6 ms, warp-local X step (a half-warp owns all rows of a group,
// shuffle-tree reduction) 19.5 ms, against 18.8 ms for the layout below.
template <int V>
struct TPCfg;
template <>
struct TPCfg<kTP32> {  // 32-column matrices: one warp holds a 32 x 32 X (R = 4)
  static constexpr int NP = 32, GX = 4, RX = 4, GV = 1, MAXT = 128, MINB = 4;
  static constexpr bool RED = true;
  static constexpr int kMaxM = kTP32MaxM;
};
template <>
struct TPCfg<kTP64> {  // 64-column matrices: 8 column groups x 16 row-threads x 4 rows; V: 2 groups x 64 rows
  static constexpr int NP = 64, GX = 8, RX = 4, GV = 2, MAXT = 128, MINB = 4;
  static constexpr bool RED = false;
  static constexpr int kMaxM = kTP64MaxM;
};

template <int V>
static size_t park_bytes_v() {
  using C = TPCfg<V>;
  return 8 * l0tp_park_elems<C::NP, C::GX, C::RX, C::GV>(tp_threads<C::NP, C::GX, C::RX, C::GV>(C::kMaxM));
}

// Sized for the largest CTA of the variant (the planner's M limit): a bucket launches every member
// with the threads of its tallest matrix, and the park layout is strided by the thread count.
size_t l0tp_park_bytes(int variant, int M) {
  (void)M;
  switch (variant) {
    case kTP32: return park_bytes_v<kTP32>();
    case kTP64: return park_bytes_v<kTP64>();
    default: return 0;
  }
}

template <typename T, int V>
static int occupancy_v(int maxM) {
  using C = TPCfg<V>;
  const int threads = tp_threads<C::NP, C::GX, C::RX, C::GV>(maxM);
  const size_t smem = l0tp_smem_bytes<T, C::NP, C::GX, C::RX, C::RED>(maxM, threads);
  auto kern = l0tp_kernel<T, C::NP, C::GX, C::RX, C::GV, C::RED, C::MAXT, C::MINB>;
  if (cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem) != cudaSuccess) return -1;
  int nb = 0;
  if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, kern, threads, smem) != cudaSuccess) return -1;
  return nb;
}

// Resident CTAs per SM of a two-phase variant for a bucket of height maxM (diagnostics).
int l0tp_occupancy(int variant, int fp32, int maxM) {
  switch (variant) {
    case kTP32: return fp32 ? occupancy_v<float, kTP32>(maxM) : occupancy_v<double, kTP32>(maxM);
    case kTP64: return fp32 ? occupancy_v<float, kTP64>(maxM) : occupancy_v<double, kTP64>(maxM);
    default: return -1;
  }
}

template <typename T, int V>
static cudaError_t launch_v(const MatDesc* descs, const int* order, int count, int maxM, const SlotPool& pool,
                            cudaStream_t stream) {
  using C = TPCfg<V>;
  return launch_tp_t<T, C::NP, C::GX, C::RX, C::GV, C::RED, C::MAXT, C::MINB>(descs, order, count, maxM, pool, stream);
}

cudaError_t launch_l0tp(int variant, int fp32, const MatDesc* descs, const int* order, int count, int maxM,
                        const SlotPool& pool, cudaStream_t stream) {
  switch (variant) {
    case kTP32:
      return fp32 ? launch_v<float, kTP32>(descs, order, count, maxM, pool, stream)
                  : launch_v<double, kTP32>(descs, order, count, maxM, pool, stream);
    case kTP64:
      return fp32 ? launch_v<float, kTP64>(descs, order, count, maxM, pool, stream)
                  : launch_v<double, kTP64>(descs, order, count, maxM, pool, stream);
    default: return cudaErrorInvalidValue;
  }
}

}  // namespace wcsvd

#ifdef WCSVD_PHASE_PROFILE
extern "C" WCSVD_API int wcsvd_debug_tp_cycles(unsigned long long* out, int reset) {
  if (cudaMemcpyFromSymbol(out, wcsvd::g_tp_cycles, sizeof(unsigned long long) * 8) != cudaSuccess) return -1;
  if (reset) {
    unsigned long long z[8] = {0, 0, 0, 0, 0, 0, 0, 0};
    cudaMemcpyToSymbol(wcsvd::g_tp_cycles, z, sizeof(z));
  }
  return 0;
}
#endif

// Diagnostics: resident CTAs per SM of the Level-0 two-phase kernel for `variant` (kernels.h) and
// matrices of height <= maxM; -1 if unknown.
extern "C" WCSVD_API int wcsvd_debug_l0tp_occupancy(int variant, int fp32, int maxM) {
  return wcsvd::l0tp_occupancy(variant, fp32, maxM);
}
