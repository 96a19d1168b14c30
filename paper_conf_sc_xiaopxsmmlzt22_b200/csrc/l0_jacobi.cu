// l0_jacobi.cu -- Level-0 batched SVD kernel: the whole one-sided Jacobi of a matrix that fits
// on-chip, in one CTA, with every sweep in-kernel and finalisation fused
// (Alg 2 l.2-3; Step 1; kernel design §IV.B).
//
// B200 design. The paper keeps the matrix in shared memory and gives each column
// pair an alpha-warp. On sm_100a an SMEM-resident sweep is bound by the 128 B/clk
// shared-memory port (every element is read and written once per step), so here the working
// matrix X (M x NP) and V (NP x NP) live in REGISTERS, distributed by rows: a thread holds R rows
// x NL = NP/G columns; G adjacent lanes share one row-group. The round-robin pairs always sit in
// fixed slot pairs (2k, 2k+1) (common.cuh), so a rotation's outputs are written straight into the
// registers of their destination slots (the column permutation is a register rename, ping-ponged
// between two arrays); only the two ring elements that cross a column-group boundary move, by one
// warp shuffle each. Per step the cross-row work is one fixed-order reduction of the partial dot
// products gamma_k = sum_r x_r,2k x_r,2k+1 (through SMEM, by one warp: lane k owns pair k) and
// one broadcast of (c_k, s_k). Norms a_i^T a_i are cached and updated by eq (6)
// in its closed form alpha' = alpha + t gamma, beta' = beta - t gamma
// (identical, since t^2 + 2 tau t - 1 = 0); they are recomputed exactly at the first step of every
// sweep; sigma is recomputed exactly at finalisation.
#include <cuda_runtime.h>

#include <cmath>

#include "common.cuh"
#include "kernels.h"
#include "prec.cuh"
#include "rotation.cuh"

namespace wcsvd {

namespace {

// Per-CTA state shared by the step functions.
template <typename T>
struct L0Ctx {
  using V2 = typename Prec<T>::V2;
  T* part;         // [2 parity][3][RW4][PS]: partial gamma / alpha / beta per (row-thread, pair)
  T* nrm;          // this warp's [2][NP] cached squared norms per slot (step parity)
  V2* cs;          // this warp's [G][LP+1] (c, s) per pair (padded against bank conflicts)
  int RW4, PS;
  int lane, g, rt;
  bool isW;
  int dtop, dbot;  // lane k: the slots that the contents of slots 2k, 2k+1 move to
  T tol2;
  int gs;          // global step counter (parity of the partial and norm buffers)
  bool rot_sweep;  // some rotation in the current sweep (identical in every warp)
};

// One round-robin step: every pair of the matrix is orthogonalised once; reads the
// slots from x, writes the rotated, moved slots to y. One CTA barrier per step: every warp reduces
// the row-thread partials itself (lane k = pair k, fixed order) and computes the same rotations,
// so the (c, s) broadcast needs no second barrier; results are bitwise identical across warps.
template <typename T, int NP, int G, int R, bool FIRST>
__device__ __forceinline__ void l0_step(L0Ctx<T>& cx, const T (&x)[R][NP / G], T (&y)[R][NP / G]) {
  using V2 = typename Prec<T>::V2;
  constexpr int NL = NP / G;
  constexpr int LP = NL / 2;
  constexpr int NPAIR = NP / 2;
  static_assert(LP >= 2 && NPAIR <= 32, "L0 tile");
  const int g = cx.g;
  const int par = cx.gs & 1;
  const int SEC = cx.RW4 * cx.PS;  // one partial section
  T* part = cx.part + par * 3 * SEC;
  // Phase 1: this thread's partial dot products for its pairs (and squared norms at sweep start).
  if (cx.isW) {
    const int base = cx.rt * cx.PS + g * LP;
#pragma unroll
    for (int j = 0; j < LP; ++j) {
      T gm = 0, al = 0, be = 0;
#pragma unroll
      for (int r = 0; r < R; ++r) {
        gm = fma(x[r][2 * j], x[r][2 * j + 1], gm);
        if (FIRST) {
          al = fma(x[r][2 * j], x[r][2 * j], al);
          be = fma(x[r][2 * j + 1], x[r][2 * j + 1], be);
        }
      }
      part[base + j] = gm;
      if (FIRST) {
        part[SEC + base + j] = al;
        part[2 * SEC + base + j] = be;
      }
    }
  }
  __syncthreads();
  // Phase 2 (every warp; lane k = pair k): fixed-order sum over row-threads, eq (4), eq (6).
  bool rot = false;
  {
    const int k = cx.lane;
    if (k < NPAIR) {
      const int PS = cx.PS;
      T g4[4] = {0, 0, 0, 0}, a4[4] = {0, 0, 0, 0}, b4[4] = {0, 0, 0, 0};
      for (int i = 0; i < cx.RW4; i += 4) {  // rows [RW, RW4) are zero
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
        al = cx.nrm[par * NP + 2 * k];
        be = cx.nrm[par * NP + 2 * k + 1];
      }
      T c, sn, t;
      rot = jacobi_rotation(al, be, gm, cx.tol2, c, sn, t);
      cx.cs[(k / LP) * (LP + 1) + (k % LP)] = Prec<T>::mk(c, sn);
      // eq (6) in closed form: alpha' = alpha + t gamma, beta' = beta - t gamma
      cx.nrm[(par ^ 1) * NP + cx.dtop] = rot ? fma(t, gm, al) : al;
      cx.nrm[(par ^ 1) * NP + cx.dbot] = rot ? fma(-t, gm, be) : be;
    }
  }
  cx.rot_sweep |= (__ballot_sync(0xffffffffu, rot) != 0u);
  __syncwarp();
  // Phase 3: rotate this thread's rows of X or V (eq 3) and move the slots (common.cuh ring).
  // Outputs of local pair j: top -> top[j+1], bot -> bot[j-1]. Group 0 keeps top[0] and sends
  // bot[0] to its top[1]; other groups receive top[0] from the left neighbour lane; the last group
  // moves its last top to its last bot, the others receive their last bot from the right.
  T top0[R], send_l[R], send_r[R];
  const V2* cs = cx.cs + g * (LP + 1);
#pragma unroll
  for (int j = 0; j < LP; ++j) {
    const V2 p = cs[j];
#pragma unroll
    for (int r = 0; r < R; ++r) {
      const T a = x[r][2 * j], b = x[r][2 * j + 1];
      // eq (3): (a^_i, a^_j) = (a_i, a_j) [[c, -s], [s, c]]
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
  ++cx.gs;
}

// One sweep of NP-1 steps starting in x; ends in y with every slot back in its original column.
template <typename T, int NP, int G, int R>
__device__ __forceinline__ void l0_sweep(L0Ctx<T>& cx, T (&x)[R][NP / G], T (&y)[R][NP / G]) {
  cx.rot_sweep = false;
  l0_step<T, NP, G, R, true>(cx, x, y);
  for (int i = 0; i < (NP - 2) / 2; ++i) {
    l0_step<T, NP, G, R, false>(cx, y, x);
    l0_step<T, NP, G, R, false>(cx, x, y);
  }
}

}  // namespace

// Shared-memory bytes of one CTA (must match the carve-up in the kernel).
template <typename T, int NP, int G, int R, bool WITHV>
size_t l0_smem_bytes(int M, int threads) {
  const int RW4 = ((M + R - 1) / R + 3) / 4 * 4;
  const int PS = NP / 2 + 1;
  const int RV = WITHV ? NP / R : RW4;  // rows of the sign-rule scratch (V rows, or X rows)
  const int LP = NP / G / 2;
  const int NW = threads / 32;
  return sizeof(T) * 6 * (size_t)RW4 * PS                              // partials, 2 parities
         + (size_t)NW * (2 * sizeof(T) * G * (LP + 1) + sizeof(T) * 2 * NP)  // per-warp cs, nrm
         + sizeof(T) * (2 * NP + (size_t)RV * NP) + sizeof(int) * (NP + 8) + 16;
}

// One CTA per matrix. Thread t: group g = t % G, row-thread rt = t / G. Row-threads [0, RW) hold
// rows rt*R .. rt*R+R-1 of X; row-threads [RW, RW+RV) hold rows of V (RV = NP/R); the rest (to a
// multiple of 32) hold zeros and only take part in shuffles.
template <typename T, int NP, int G, int R, int MAXT, bool WITHV>
__global__ void __launch_bounds__(MAXT) l0_jacobi_kernel(const MatDesc* __restrict__ descs,
                                                        const int* __restrict__ order) {
  // T: arithmetic and I/O type (double for wcsvd_batched, float for wcsvd_batched_f32).
  using V2 = typename Prec<T>::V2;
  constexpr int NL = NP / G;
  constexpr int LP = NL / 2;
  constexpr int NPAIR = NP / 2;
  constexpr int RV = WITHV ? NP / R : 0;  // V row-threads (none in the values / U-only mode, §8(f4))
  const MatDesc d = descs[order[blockIdx.x]];
  const int M = d.M, N = d.N;
  const int RW = (M + R - 1) / R;
  const int PS = NPAIR + 1;  // odd stride (doubles): conflict-free partial writes and reads
  const int NT = blockDim.x;
  const int tid = threadIdx.x;
  const int g = tid % G;
  const int rt = tid / G;
  const bool isW = rt < RW;
  const bool isV = !isW && rt < RW + RV;

  extern __shared__ __align__(16) unsigned char smem_raw[];
  const int RW4 = (RW + 3) / 4 * 4;  // partial rows padded to 4 (zeros)
  const int NWARP = NT / 32;
  unsigned long long* s_max = reinterpret_cast<unsigned long long*>(smem_raw);  // [2] (16 B)
  T* s_part = reinterpret_cast<T*>(smem_raw + 16);                        // [2][3][RW4][PS]
  V2* s_csw = reinterpret_cast<V2*>(s_part + 6 * RW4 * PS);               // [NWARP][G][LP+1]
  T* s_nrmw = reinterpret_cast<T*>(s_csw + NWARP * G * (LP + 1));         // [NWARP][2][NP]
  T* s_sig = s_nrmw + NWARP * 2 * NP;                                     // [NP]
  T* s_sgn = s_sig + NP;                                                  // [NP]
  const int SR = WITHV ? RV : RW4;                                        // sign-rule rows
  T* s_vbest = s_sgn + NP;                                                // [SR][NP]
  int* s_rank = reinterpret_cast<int*>(s_vbest + SR * NP);                // [NP]
  int* s_flags = s_rank + NP;                                             // [8]
  if (tid < 4) s_flags[tid] = 0;
  if (tid == 0) *s_max = 0ull;
  for (int e = tid; e < 6 * RW4 * PS; e += NT) s_part[e] = T(0);
  __syncthreads();

  // ---- Stage-in: X = A (m >= n) or A^T (m < n), zero-padded; V = I. ----
  T xa[R][NL], xb[R][NL];
  bool bad = false;
  T amax = 0;
  const T* Ain = reinterpret_cast<const T*>(d.A);
#pragma unroll
  for (int r = 0; r < R; ++r) {
#pragma unroll
    for (int l = 0; l < NL; ++l) {
      const int col = g * NL + l;
      T v = 0;
      if (isW) {
        const int row = rt * R + r;
        if (row < M && col < N) {
          v = d.swapped ? Ain[(size_t)row * d.lda + col] : Ain[(size_t)col * d.lda + row];
          bad |= !isfinite(v);
          amax = fmax(amax, fabs(v));
        }
      } else if (isV) {
        v = ((rt - RW) * R + r == col) ? T(1) : T(0);
      }
      xa[r][l] = v;
    }
  }
  if (bad) atomicOr(&s_flags[2], 1);
  if (isW && amax > T(0)) atomicMax(s_max, (unsigned long long)__double_as_longlong((double)amax));
  __syncthreads();
  const bool nonfinite = s_flags[2] != 0;
  // Exact power-of-two pre-scaling to max|x| in [0.5, 1): every product in the iteration stays in
  // range, and (no under/overflow) the rotations, U and V are bitwise those of the unscaled input
  // (SURVEY P10); sigma is scaled back at finalisation.
  int sexp = 0;
  if (!nonfinite && *s_max != 0ull) {
    frexp(__longlong_as_double((long long)*s_max), &sexp);
    if (isW) {
      const T f = (T)ldexp(1.0, -sexp);
#pragma unroll
      for (int r = 0; r < R; ++r)
#pragma unroll
        for (int l = 0; l < NL; ++l) xa[r][l] *= f;
    }
  }

  const int lane = tid & 31, warp = tid >> 5;
  L0Ctx<T> cx;
  cx.part = s_part;
  cx.nrm = s_nrmw + warp * 2 * NP;
  cx.cs = s_csw + warp * G * (LP + 1);
  cx.RW4 = RW4;
  cx.PS = PS;
  cx.lane = lane;
  cx.g = g;
  cx.rt = rt;
  cx.isW = isW;
  cx.dtop = rr_dest(2 * lane, NP);
  cx.dbot = rr_dest(2 * lane + 1, NP);
  cx.tol2 = (T)(d.tol * d.tol);
  cx.gs = 0;
  cx.rot_sweep = false;
  int sweep = 0;
  bool converged = false;
  bool in_b = false;
  if (!nonfinite) {
    for (;;) {
      l0_sweep<T, NP, G, R>(cx, xa, xb);  // ends in xb
      ++sweep;
      if (!cx.rot_sweep) { converged = true; in_b = true; break; }
      if (sweep >= d.max_sweeps) { in_b = true; break; }
      l0_sweep<T, NP, G, R>(cx, xb, xa);  // ends in xa
      ++sweep;
      if (!cx.rot_sweep) { converged = true; break; }
      if (sweep >= d.max_sweeps) break;
    }
  }
  if (in_b) {
#pragma unroll
    for (int r = 0; r < R; ++r)
#pragma unroll
      for (int l = 0; l < NL; ++l) xa[r][l] = xb[r][l];
  }

  // ---- Finalisation: sigma_j = ||x_j|| (fresh, fixed order), stable descending
  // rank (Z15), U = X / sigma, sign rule on the square factor V_x (Z15), un-orientation.
  __syncthreads();
  if (isW) {
#pragma unroll
    for (int l = 0; l < NL; ++l) {
      T a = 0;
#pragma unroll
      for (int r = 0; r < R; ++r) a = fma(xa[r][l], xa[r][l], a);
      const int col = g * NL + l;  // [RW][NP] view over the first two partial sections
      s_part[(col < NPAIR ? 0 : RW4) * PS + rt * PS + (col % NPAIR)] = a;
    }
  }
  // Z15 sign rule: the largest-|.| entry (first on ties) of each column of the square factor V_x is
  // made positive; without V (values / U-only mode) the rule is applied to the columns of X instead.
  if (WITHV ? isV : isW) {
#pragma unroll
    for (int l = 0; l < NL; ++l) {
      T best = 0;
#pragma unroll
      for (int r = 0; r < R; ++r)
        if (fabs(xa[r][l]) > fabs(best)) best = xa[r][l];
      s_vbest[(rt - (WITHV ? RW : 0)) * NP + g * NL + l] = best;
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
    for (int i = 0; i < (WITHV ? RV : RW); ++i) {
      const T v = s_vbest[i * NP + j];
      if (fabs(v) > fabs(best)) best = v;
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
    for (int l = 0; l < NL; ++l) {
      const int col = g * NL + l;
      if (col < N) {
        const int rk = s_rank[col];
        const T sj = s_sig[col];
        const T sgn = s_sgn[col];
        const bool ok = sj > thresh;
        needs_completion |= !ok;
#pragma unroll
        for (int r = 0; r < R; ++r) {
          const int row = rt * R + r;
          if (row < M)  // rank-deficient columns: signed zero, completed by complete_u_kernel
            dstW[(size_t)rk * ldW + row] = nonfinite ? nanv : (ok ? sgn * (xa[r][l] / sj) : sgn * T(0));
        }
      }
    }
  }
  if (isV && dstV) {
#pragma unroll
    for (int l = 0; l < NL; ++l) {
      const int col = g * NL + l;
      if (col < N) {
        const int rk = s_rank[col];
        const T sgn = s_sgn[col];
#pragma unroll
        for (int r = 0; r < R; ++r) {
          const int vrow = (rt - RW) * R + r;
          if (vrow < N) dstV[(size_t)rk * ldV + vrow] = nonfinite ? nanv : sgn * xa[r][l];
        }
      }
    }
  }
  if (needs_completion && !nonfinite) atomicOr(&s_flags[3], 1);
  T* Sout = reinterpret_cast<T*>(d.S);
  for (int j = tid; j < N; j += NT) Sout[s_rank[j]] = nonfinite ? nanv : (T)ldexp((double)s_sig[j], sexp);
  __syncthreads();
  if (tid == 0) {
    if (d.info) d.info[d.idx] = nonfinite ? -2 : (converged ? sweep : -1);
    if (d.sweeps_inner) d.sweeps_inner[d.idx] = 0;
    if (d.status) d.status[d.idx] = (s_flags[3] && dstW) ? kNeedsCompletion : 0;
  }
}

// ---- launcher ----
template <typename T, int NP, int G, int R, int MAXT, bool WITHV>
static cudaError_t launch_l0_t(const MatDesc* descs, const int* order, int count, int maxM,
                               cudaStream_t stream) {
  const int RW = (maxM + R - 1) / R;
  int threads = (RW + (WITHV ? NP / R : 0)) * G;
  threads = (threads + 31) / 32 * 32;
  if (threads > MAXT) return cudaErrorInvalidConfiguration;
  const size_t smem = l0_smem_bytes<T, NP, G, R, WITHV>(maxM, threads);
  auto kern = l0_jacobi_kernel<T, NP, G, R, MAXT, WITHV>;
  cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  kern<<<count, threads, smem, stream>>>(descs, order);
  return cudaGetLastError();
}

template <typename T, bool WITHV>
static cudaError_t launch_l0_v(int variant, const MatDesc* descs, const int* order, int count, int maxM,
                               cudaStream_t stream) {
  switch (variant) {
    case kL0_8:   return launch_l0_t<T, 8, 1, 8, 256, WITHV>(descs, order, count, maxM, stream);
    case kL0_16:  return launch_l0_t<T, 16, 2, 8, 256, WITHV>(descs, order, count, maxM, stream);
    case kL0_32:  return launch_l0_t<T, 32, 2, 4, 256, WITHV>(descs, order, count, maxM, stream);
    case kL0_32s: return launch_l0_t<T, 32, 2, 1, 512, WITHV>(descs, order, count, maxM, stream);
    case kL0_48:  return launch_l0_t<T, 48, 2, 2, 256, WITHV>(descs, order, count, maxM, stream);
    case kL0_64:  return launch_l0_t<T, 64, 8, 8, 256, WITHV>(descs, order, count, maxM, stream);
    default: return cudaErrorInvalidValue;
  }
}

// Variant table (planner ids). E = R * NP / G elements per thread. withv = 0: V_x is not accumulated
// (it is not requested; §8(f4) values / U-only mode) -- half the threads and registers per matrix.
// fp32 = 1: the fp32 variant (§8(f1)), iterated in float.
cudaError_t launch_l0(int variant, int withv, int fp32, const MatDesc* descs, const int* order, int count,
                      int maxM, cudaStream_t stream) {
  if (fp32)
    return withv ? launch_l0_v<float, true>(variant, descs, order, count, maxM, stream)
                 : launch_l0_v<float, false>(variant, descs, order, count, maxM, stream);
  return withv ? launch_l0_v<double, true>(variant, descs, order, count, maxM, stream)
               : launch_l0_v<double, false>(variant, descs, order, count, maxM, stream);
}

}  // namespace wcsvd
