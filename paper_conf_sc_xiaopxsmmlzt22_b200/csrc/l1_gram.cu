// l1_gram.cu -- Level-1 block one-sided Jacobi over column-block pairs, Gram path:
// (1) Gram B_ij = A_ij^T A_ij, (2) threshold Jacobi EVD of B_ij in shared memory / registers,
// (3) GEMM update A_ij <- A_ij J_ij and V_ij <- V_ij J_ij, (4) off-norm test -- Alg 1 l.5-7
// (PAPER.md:68-70), Alg 2 l.10-11 + l.16, Step 2, the parallel
// EVD of §IV.C and the two batched GEMMs of §IV.D.
//
// B200 design: one CTA per matrix runs every sweep in-kernel (no host round
// trip); each warp owns one column-block pair of the current round-robin step at a
// time; a CTA barrier separates steps. The working copy W (m_pad x n_pad) and V live in global
// memory (L2-resident while the CTA works on them). Both contractions use FP64 DMMA.8x8x4 tiles
// fed straight from L2 into registers (no SMEM staging needed: each fragment load is 8 columns x
// 32 contiguous bytes); the Gram computes only the upper tiles. The EVD is the paper's parallel
// two-sided Jacobi with round-robin pairs: B stays in SMEM in original index
// order and is updated in 2x2 quads; J is accumulated in registers (row x of J in lane x) in
// "slot" order so that every rotation writes fixed registers (common.cuh). Threshold rotations make
// J = I exactly once B is diagonal to tol; the EVD is capped at inner_cap sweeps
// (Z8); J is re-orthogonalised by one Newton-Schulz step J <- J - J (J^T J - I)/2 before it is
// applied (Z9(ii); R-NS: a build option keeps it off). A pair whose Gram is already diagonal to tol is skipped with no writes; a
// sweep in which every pair is skipped ends the iteration (Z6, Z9(iii)).
#include <cuda_runtime.h>

#include <cmath>

#include "common.cuh"
#include "dmma.cuh"
#include "kernels.h"
#include "rotation.cuh"
#include "wcsvd.h"

// Newton-Schulz cleanup of J before it is applied. -DWCSVD_L1_NS=0 drops it (ablation,
// DESIGN.md §3 R-NS): 4-5% faster on Level 1 (B200, r01g: C3 229 -> 220 ms, C4 364 -> 345 ms, C5 2.93 ->
// 2.82 s) but sigma / residual errors ~50x larger on the Table VII stand-ins (up to 5.5e-13 / 9.3e-13 on
// the W-cycle, against the 1e-12 bar), so the default keeps it.
#ifndef WCSVD_L1_NS
#define WCSVD_L1_NS 1
#endif
// fp64 inner EVD storage: 1 = full symmetric B, select-free quads (evd_step_full), 0 = upper triangle in
// the swizzled slot layout (evd_step; round-1 kernel, A/B builds)
#ifndef WCSVD_EVD_FULL
#define WCSVD_EVD_FULL 1
#endif
// Nearly diagonal pair Grams (R-PERT): when every rotating b_pq is below kPertDelta times
// |b_pp - b_qq|, J is the first-order eigenvector matrix I + E (E_pq = b_pq / (b_qq - b_pp)) made
// orthogonal by two Newton-Schulz steps, instead of the 2w-1-step Jacobi sweep. 0 disables it.
#ifndef WCSVD_L1_PERT
#define WCSVD_L1_PERT 1
#endif
// (delta = 1e-3 with three Newton-Schulz steps covers more pairs but measured slower: C3 211.4 vs 208.6
// ms, 12.39 vs 12.37 sweeps; half C5 1417 vs 1413 ms)
#ifndef WCSVD_L1_PERT_DELTA
#define WCSVD_L1_PERT_DELTA 1e-4
#endif
constexpr double kPertDelta = WCSVD_L1_PERT_DELTA;
// Newton-Schulz steps after J = I + E: ||J^T J - I|| <= (2w delta)^2 shrinks as e -> 0.75 e^2 per step
constexpr int kPertNS = kPertDelta <= 1e-4 ? 2 : 3;
// Inner EVD angle: 0 = exact fp64 eq (4) (R-ROT), 1 = fp32 angle with fp64-orthogonal (c, s) (R-ROT32)
#ifndef WCSVD_EVD_ROT32
#define WCSVD_EVD_ROT32 0
#endif
// Resident CTAs per SM the Level-1 kernels are compiled for (register budget 65536 / (32 NW minB)).
#ifndef WCSVD_L1_MINB
#define WCSVD_L1_MINB(nw) 1
#endif
#ifndef WCSVD_L1_NSTAGE
#define WCSVD_L1_NSTAGE 3
#endif

namespace wcsvd {

namespace {

#ifdef WCSVD_PHASE_PROFILE
// Debug builds only (-DWCSVD_PHASE_PROFILE): per-phase clock64() totals, lane 0 of every warp.
__device__ unsigned long long g_phase_cycles[12];
#define PHASE_T0() long long _pt = clock64()
#define PHASE_MARK(i)                                                        \
  do {                                                                       \
    long long _pn = clock64();                                               \
    if ((threadIdx.x & 31) == 0) atomicAdd(&g_phase_cycles[i], (unsigned long long)(_pn - _pt)); \
    _pt = _pn;                                                               \
  } while (0)
#define PHASE_COUNT(i)                                                       \
  do {                                                                       \
    if ((threadIdx.x & 31) == 0) atomicAdd(&g_phase_cycles[i], 1ull);        \
  } while (0)
#else
#define PHASE_T0() (void)0
#define PHASE_MARK(i) (void)0
#define PHASE_COUNT(i) (void)0
#endif

// Named barrier over `count` threads (whole warps). The non-.aligned form (barrier.sync, not bar.sync):
// the two warps of a split pair group reach it from different code (process_pair_split<0> / <1>), which
// the .aligned form does not allow; the warp is reconverged first (lane-0-only spins precede some uses).
__device__ __forceinline__ void named_bar(int id, int count) {
  __syncwarp();
  asm volatile("barrier.sync %0, %1;" ::"r"(id), "r"(count) : "memory");
}

template <int W2>
struct PairCfg {
  static constexpr int W = W2 / 2;          // block width w
  static constexpr int CG = W2 / 8;         // 8-column groups per pair panel
  static constexpr int NTU = CG * (CG + 1) / 2;  // upper tiles of the 2w x 2w Gram
  // SMEM row stride of the 2w x 2w J / E / J' buffers (doubles). W2 + 3: the Newton-Schulz fragment
  // loads ((8i + l/4) BS + 4kk + l%4 and (4kk + l%4) BS + 8j + l/4), the J' stores and the J staging
  // stores take 3 / 3 / 3 / 2 wavefronts per warp access instead of 4 / 4 / 4 / 2 with W2 + 1 (bank
  // model in DESIGN.md §5.2); the EVD's full-symmetric B uses its own stride W2.
  static constexpr int BS = W2 + 3;
  static_assert(W2 == 16 || W2 == 32, "pair panel width");
};

// Per-warp SMEM region.
template <int W2>
struct WarpSmem {
  double* B;    // [W2][BS] Gram / E = J^T J - I / J'
  double* S;    // [W2][BS] staged J
  double2* cs;  // [NPR]    (c, s) of the step's rotations
  double* tt;   // [NPR]    t of the step's rotations (0 = none)
  int2* pq;     // [NPR]    (p, q) original indices of the step's pairs
  double* ring;  // [NSTAGE][W2][SL] cp.async slab ring for the Gram / update panels (aliases B, S)
  static constexpr int SL = 20;      // ring column stride (doubles): 16 rows + 4 pad (conflict-free fragments)
  static constexpr int NSTAGE = WCSVD_L1_NSTAGE;  // slabs in flight (ring stages)
  static constexpr int SLAB = W2 * SL;  // doubles per slab
  __host__ __device__ static constexpr size_t region() {
    return (2 * W2 * PairCfg<W2>::BS > NSTAGE * SLAB ? 2 * W2 * PairCfg<W2>::BS : NSTAGE * SLAB) * sizeof(double);
  }
  __host__ __device__ static constexpr size_t bytes() {
    return region() + (sizeof(double2) + sizeof(double) + sizeof(int2)) * (W2 / 2);
  }
};

// P column j (0 <= j < 2w) of pair (I, J) -> working-matrix column.
template <int W2>
__device__ __forceinline__ int pcol(int j, int I, int J) {
  constexpr int W = W2 / 2;
  return (j < W) ? I * W + j : J * W + (j - W);
}

// Upper tiles of P^T P for a panel whose 8-col groups start at ptr[c] (already offset by lane:
// column 8c + lane/4, row lane%4); `rows` multiple of 16; `rstride` = element stride per row.
template <int W2>
__device__ __forceinline__ void gram_load(double (&f)[4][W2 / 8], const double* const (&ptr)[W2 / 8], int r0,
                                          int rstride) {
#pragma unroll
  for (int u = 0; u < 4; ++u)
#pragma unroll
    for (int c = 0; c < W2 / 8; ++c) f[u][c] = ptr[c][(size_t)(r0 + 4 * u) * rstride];
}

template <int W2>
__device__ __forceinline__ void gram_mma(double (&acc)[PairCfg<W2>::NTU][2], const double (&f)[4][W2 / 8]) {
  constexpr int CG = W2 / 8;
#pragma unroll
  for (int u = 0; u < 4; ++u) {
    int t = 0;
#pragma unroll
    for (int a = 0; a < CG; ++a)
#pragma unroll
      for (int b = a; b < CG; ++b) dmma884(acc[t++], f[u][a], f[u][b]);
  }
}

// Upper tiles of P^T P for a panel whose 8-col groups start at ptr[c] (already offset by lane:
// column 8c + lane/4, row lane%4); `rows` multiple of 16; `rstride` = element stride per row.
// The next 16-row slab is loaded while the current one feeds the DMMAs (register ping-pong).
template <int W2>
__device__ __forceinline__ void gram_tiles(const double* const (&ptr)[W2 / 8], int rows, int rstride,
                                           double (&acc)[PairCfg<W2>::NTU][2]) {
  constexpr int CG = W2 / 8;
#pragma unroll
  for (int t = 0; t < PairCfg<W2>::NTU; ++t) acc[t][0] = acc[t][1] = 0.0;
  double f0[4][CG], f1[4][CG];
  gram_load<W2>(f0, ptr, 0, rstride);
  for (int r0 = 0;;) {
    if (r0 + 16 < rows) gram_load<W2>(f1, ptr, r0 + 16, rstride);
    gram_mma<W2>(acc, f0);
    if ((r0 += 16) >= rows) break;
    if (r0 + 16 < rows) gram_load<W2>(f0, ptr, r0 + 16, rstride);
    gram_mma<W2>(acc, f1);
    if ((r0 += 16) >= rows) break;
  }
}

// ---- cp.async slab pipeline (per warp): 16-row x 2w-column panel slabs, global -> SMEM ring ----
__device__ __forceinline__ void cp_async16(void* smem, const void* gmem) {
  const unsigned sa = (unsigned)__cvta_generic_to_shared(smem);
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(sa), "l"(gmem) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_async_wait() { asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory"); }

// L2 eviction priorities of the panel streams (WCSVD_L2HINT). The A panel a pair's Gram
// reads is read again by the same pair's update one EVD later (short reuse); the V panel is touched
// once per pair and next only one step later (long reuse). Hint kinds: 0 = the Gram's A loads, 1 = the
// update's A loads / stores, 2 = the update's V loads / stores. Mode 0 = no hints (plain cp.async.cg /
// st.global.cg). Measured (same box, ms, C3 / C4 / half of C5): none 226.1 / 339.0 / 1444; 1 (Gram A
// evict_last, V evict_first) 219.6 / 340.7 / 1447; 2 (1 + update A loads evict_first) 222.2 / 340.6 /
// 1452; 3 (2 + update A stores evict_last) 219.6 / 340.1 / 1446; 4 (V evict_first only) 219.6 / 339.7 /
// 1450; C4 DRAM bytes unchanged (1.51 TB per launch) in every mode: at 2w = 32 the pair's working sets
// in flight (8 per SM) exceed L2 whatever the priorities. Default 4: the V stream gives way.
#ifndef WCSVD_L2HINT
#define WCSVD_L2HINT 4
#endif
__device__ __forceinline__ unsigned long long l2_policy(int prio) {  // 0 evict_first, 1 normal, 2 evict_last
  unsigned long long p;
  if (prio == 0) asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
  else if (prio == 2) asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
  else asm volatile("createpolicy.fractional.L2::evict_normal.b64 %0, 1.0;" : "=l"(p));
  return p;
}
// priority of loads (LD) or stores (ST) of hint kind K under WCSVD_L2HINT
template <int K, bool ST>
__device__ __forceinline__ constexpr int l2_prio() {
#if WCSVD_L2HINT == 1
  return K == 0 ? 2 : (K == 2 ? 0 : 1);
#elif WCSVD_L2HINT == 2
  return K == 0 ? 2 : (K == 2 ? 0 : (ST ? 1 : 0));
#elif WCSVD_L2HINT == 3
  return K == 0 ? 2 : (K == 2 ? 0 : (ST ? 2 : 0));
#elif WCSVD_L2HINT == 4
  return K == 2 ? 0 : 1;
#else
  return -1;
#endif
}
__device__ __forceinline__ void cp_async16_hint(void* smem, const void* gmem, unsigned long long pol) {
  const unsigned sa = (unsigned)__cvta_generic_to_shared(smem);
  asm volatile("cp.async.cg.shared.global.L2::cache_hint [%0], [%1], 16, %2;" ::"r"(sa), "l"(gmem), "l"(pol) : "memory");
}
__device__ __forceinline__ void st_hint(double* p, double v, unsigned long long pol) {
  asm volatile("st.global.L2::cache_hint.f64 [%0], %1, %2;" ::"l"(p), "d"(v), "l"(pol) : "memory");
}

// Chunk addressing of a pair panel (2w columns = block I's w columns, then block J's): lane's chunk i
// (W2/4 chunks of 16 B per lane and slab) is column c = lane/8 + 4i, i.e. block I for i < W2/8, block J
// after, so two element offsets and 4 ld describe every chunk (instead of W2/4 registers).
struct PanelAddr {
  int aI, aJ;  // element offsets of this lane's first chunk column in block I / block J (+ row 2h)
  int ld4;     // 4 ld
};
template <int W2>
__device__ __forceinline__ PanelAddr panel_addr(int I, int J, int ld, int lane) {
  constexpr int W = W2 / 2;
  const int c0 = lane >> 3, h = lane & 7;
  return PanelAddr{(I * W + c0) * ld + 2 * h, (J * W + c0) * ld + 2 * h, 4 * ld};
}

// Issue the copy of rows [r0, r0+16) of the 2w panel columns into ring stage `st`: W2 x 8 chunks of
// 16 B, W2/4 per lane.
template <int W2, int K = 1>
__device__ __forceinline__ void slab_issue(double* ring, const double* base, const PanelAddr& pa, int r0, int st,
                                           int lane, unsigned long long pol = 0ull) {
  constexpr int SL = WarpSmem<W2>::SL, HI = W2 / 8;
  double* dst = ring + st * WarpSmem<W2>::SLAB + (lane >> 3) * SL + 2 * (lane & 7);
#pragma unroll
  for (int i = 0; i < W2 / 4; ++i) {
    const int off = (i < HI ? pa.aI + i * pa.ld4 : pa.aJ + (i - HI) * pa.ld4) + r0;
    if constexpr (l2_prio<K, false>() >= 0) cp_async16_hint(dst + 4 * i * SL, base + off, pol);
    else cp_async16(dst + 4 * i * SL, base + off);
  }
}

// Upper tiles of P^T P for the global panel of pair (I, J): slabs stream through the NS-stage ring
// while the DMMAs consume the previous ones (no register staging, NS-1 slabs in flight).
template <int W2, int NS>
__device__ __forceinline__ void gram_tiles_async(double* ring, const double* base, int ld, int rows, int I, int J,
                                                 int lane, double (&acc)[PairCfg<W2>::NTU][2]) {
  constexpr int CG = W2 / 8, SL = WarpSmem<W2>::SL;
#pragma unroll
  for (int t = 0; t < PairCfg<W2>::NTU; ++t) acc[t][0] = acc[t][1] = 0.0;
  const PanelAddr pa = panel_addr<W2>(I, J, ld, lane);
  const int nslab = rows >> 4;
  const unsigned long long pol = l2_prio<0, false>() >= 0 ? l2_policy(l2_prio<0, false>()) : 0ull;
#pragma unroll
  for (int j = 0; j < NS - 1; ++j) {
    if (j < nslab) slab_issue<W2, 0>(ring, base, pa, 16 * j, j, lane, pol);
    cp_async_commit();
  }
  const int fo = (lane >> 2) * SL + (lane & 3);  // fragment offset inside a column group
  for (int sl = 0; sl < nslab; ++sl) {
    if (sl + NS - 1 < nslab) slab_issue<W2, 0>(ring, base, pa, 16 * (sl + NS - 1), (sl + NS - 1) % NS, lane, pol);
    cp_async_commit();
    cp_async_wait<NS - 1>();
    __syncwarp();
    const double* st = ring + (sl % NS) * WarpSmem<W2>::SLAB;
    double f[4][CG];
#pragma unroll
    for (int u = 0; u < 4; ++u)
#pragma unroll
      for (int c = 0; c < CG; ++c) f[u][c] = st[8 * c * SL + fo + 4 * u];
    gram_mma<W2>(acc, f);
    __syncwarp();
  }
}

// X <- X * J' for the global panel of pair (I, J), slabs streamed through the NS-stage ring; results
// are stored straight to global memory (rows of a slab are read before they are overwritten).
template <int W2, int NS, int K = 1>
__device__ __forceinline__ void apply_rotation_async(double* ring, double* base, int ld, int rows, int I, int J,
                                                     int lane, const double (&jf)[W2 / 4][W2 / 8]) {
  constexpr int CG = W2 / 8, KK = W2 / 4, SL = WarpSmem<W2>::SL;
  const PanelAddr pa = panel_addr<W2>(I, J, ld, lane);
  // output element offsets: column 8 nb + 2 (lane % 4) + e of the panel, row lane / 4 (+ 8h, + 16 sl)
  constexpr int W = W2 / 2, HB = CG / 2;
  const int oI = (I * W + 2 * (lane & 3)) * ld + (lane >> 2), oJ = (J * W + 2 * (lane & 3)) * ld + (lane >> 2);
  const int nslab = rows >> 4;
  const unsigned long long pol = l2_prio<K, false>() >= 0 ? l2_policy(l2_prio<K, false>()) : 0ull;
  const unsigned long long pst = l2_prio<K, true>() >= 0 ? l2_policy(l2_prio<K, true>()) : 0ull;
#pragma unroll
  for (int j = 0; j < NS - 1; ++j) {
    if (j < nslab) slab_issue<W2, K>(ring, base, pa, 16 * j, j, lane, pol);
    cp_async_commit();
  }
  const int fo = (lane & 3) * SL + (lane >> 2);  // A fragment: row l/4, column l%4
  for (int sl = 0; sl < nslab; ++sl) {
    if (sl + NS - 1 < nslab) slab_issue<W2, K>(ring, base, pa, 16 * (sl + NS - 1), (sl + NS - 1) % NS, lane, pol);
    cp_async_commit();
    cp_async_wait<NS - 1>();
    __syncwarp();
    const double* st = ring + (sl % NS) * WarpSmem<W2>::SLAB;
#pragma unroll
    for (int h = 0; h < 2; ++h) {
      double a[KK];
#pragma unroll
      for (int kk = 0; kk < KK; ++kk) a[kk] = st[4 * kk * SL + fo + 8 * h];
      double acc[CG][2];
#pragma unroll
      for (int nb = 0; nb < CG; ++nb) acc[nb][0] = acc[nb][1] = 0.0;
#pragma unroll
      for (int kk = 0; kk < KK; ++kk)
#pragma unroll
        for (int nb = 0; nb < CG; ++nb) dmma884(acc[nb], a[kk], jf[kk][nb]);
#pragma unroll
      for (int nb = 0; nb < CG; ++nb)
#pragma unroll
        for (int e = 0; e < 2; ++e) {
          double* dst = base + (nb < HB ? oI + (8 * nb + e) * ld : oJ + (8 * (nb - HB) + e) * ld) + 16 * sl + 8 * h;
          if constexpr (l2_prio<K, true>() >= 0) st_hint(dst, acc[nb][e], pst);
          else __stcg(dst, acc[nb][e]);
        }
    }
    __syncwarp();
  }
}

// Write upper tiles (and their mirrors) into a [W2][BS] SMEM buffer; subtract `diag_sub` on the
// diagonal (1.0 for E = J^T J - I, 0.0 for the Gram).
template <int W2>
__device__ __forceinline__ void store_sym(double* buf, const double (&acc)[PairCfg<W2>::NTU][2],
                                          int lane, double diag_sub) {
  constexpr int CG = W2 / 8, BS = PairCfg<W2>::BS;
  int t = 0;
#pragma unroll
  for (int a = 0; a < CG; ++a)
#pragma unroll
    for (int b = a; b < CG; ++b, ++t)
#pragma unroll
      for (int e = 0; e < 2; ++e) {
        const int row = 8 * a + (lane >> 2), col = 8 * b + 2 * (lane & 3) + e;
        const double v = acc[t][e] - ((row == col) ? diag_sub : 0.0);
        buf[row * BS + col] = v;
        if (a != b) buf[col * BS + row] = v;
      }
}

// ---- Inner EVD storage: B in "slot" order, moved along with the round-robin ring ----
// B (symmetric, 2w x 2w) is kept as its upper triangle indexed by *slot*: the pair k of every step
// is always slots (2k, 2k+1), so the elements a lane reads (its 2x2 quads) sit at the same
// addresses at every step; the rotated values are written straight to the slots their rows and
// columns move to (common.cuh rr_dest), into a second buffer (ping-pong). After 2w-1 steps every
// index is back in its own slot. Element (a, b), a <= b, lives at a*W2 + (b ^ ((a >> 1) & (w-1))):
// the XOR swizzle spreads each step's 32 lanes over the shared-memory banks (the two elements of a
// quad row stay one aligned 16-byte pair, loaded as one double2).
template <int W2>
__host__ __device__ __forceinline__ int evd_phys(int a, int b) {
  return a * W2 + (b ^ ((a >> 1) & (W2 / 2 - 1)));
}
template <int W2>
__device__ __forceinline__ int evd_phys_sym(int a, int b) {
  return (a <= b) ? evd_phys<W2>(a, b) : evd_phys<W2>(b, a);
}

// Lane-static EVD work map. Lane L (of the NLANES lanes working on one EVD) works for pair
// k = L mod (w) (it evaluates that pair's rotation, redundantly with the other lanes of the same k)
// and owns the off-diagonal quads {k, (k+d) mod w} for its share of d = 1 .. w/2 (d = w/2 only from
// the lower k, so every unordered pair of pairs is owned exactly once). Offsets are element offsets
// into a buffer.
template <int W2, int NLANES = 32>
struct EvdMap {
  static constexpr int NPR = W2 / 2, LPP = NLANES / NPR, HALF = NPR / 2;
  static constexpr int QPL = (HALF + LPP - 1) / LPP;  // quads per lane
  int q[QPL];       // bits 0-10 load offset (row 2lo, aligned column pair), 11 swap, 12 own-is-lo,
                    // 13 valid, 16-19 partner pair
  int st[QPL][2];   // store offsets of e00 | e01 << 16 and e10 | e11 << 16
  int dld01, dld2;  // diagonal block loads: (2k,2k) | (2k+1,2k+1) << 16, (2k,2k+1)
  int dst01, dst2;  // diagonal block stores (moved slots)
  __device__ __forceinline__ void init(int lane) {
    const int k = lane & (NPR - 1), h = lane / NPR;
#pragma unroll
    for (int i = 0; i < QPL; ++i) {
      const int d = 1 + h * QPL + i;
      const bool valid = d < HALF || (d == HALF && k < HALF);
      const int l = (k + d) & (NPR - 1), lo = min(k, l), hi = max(k, l);
      q[i] = 0;
      st[i][0] = st[i][1] = 0;
      if (!valid) continue;
      q[i] = (2 * lo * W2 + ((2 * hi) ^ (lo & ~1))) | ((lo & 1) << 11) | ((k < l) << 12) | (1 << 13) | (l << 16);
      int o[4];
#pragma unroll
      for (int e = 0; e < 4; ++e) o[e] = evd_phys_sym<W2>(rr_dest(2 * lo + (e >> 1), W2), rr_dest(2 * hi + (e & 1), W2));
      st[i][0] = o[0] | (o[1] << 16);
      st[i][1] = o[2] | (o[3] << 16);
    }
    dld01 = evd_phys<W2>(2 * k, 2 * k) | (evd_phys<W2>(2 * k + 1, 2 * k + 1) << 16);
    dld2 = evd_phys<W2>(2 * k, 2 * k + 1);
    const int a0 = rr_dest(2 * k, W2), a1 = rr_dest(2 * k + 1, W2);
    dst01 = evd_phys<W2>(a0, a0) | (evd_phys<W2>(a1, a1) << 16);
    dst2 = evd_phys_sym<W2>(a0, a1);
  }
};

// One inner EVD step (round-robin over 2w indices): every lane evaluates the rotation
// of its pair k = (slots 2k, 2k+1) from the diagonal block; lanes k < w publish (c, s) and write the
// annihilated diagonal block (eq 6 analogue, exact zero off-diagonal); every off-diagonal quad of
// B' = G^T B G is updated from one load per quad row and written, like the
// diagonal blocks, to the slots its indices move to in Bn; J <- J G in slot order (x -> y rename).
// A step in which no pair rotates only moves B and J.
template <typename T> struct Vec2;
template <> struct Vec2<double> { using type = double2; };
template <> struct Vec2<float> { using type = float2; };

template <int W2, typename T = double>
__device__ __forceinline__ bool evd_step(const T* __restrict__ Bc, T* __restrict__ Bn, typename Vec2<T>::type* cs,
                                         const EvdMap<W2>& em, int lane, T tol2, const T (&x)[W2], T (&y)[W2]) {
  using T2 = typename Vec2<T>::type;
  constexpr int NPR = W2 / 2, QPL = EvdMap<W2>::QPL;
  const T bpp = Bc[em.dld01 & 0xffff], bqq = Bc[em.dld01 >> 16], bpq = Bc[em.dld2];
  T c, s, t;
  const bool rot = jacobi_rotation(bpp, bqq, bpq, tol2, c, s, t);
  if (lane < NPR) {
    cs[lane] = T2{c, s};
    Bn[em.dst01 & 0xffff] = rot ? fma(t, bpq, bpp) : bpp;
    Bn[em.dst01 >> 16] = rot ? fma(-t, bpq, bqq) : bqq;
    Bn[em.dst2] = rot ? T(0) : bpq;
  }
  T b00[QPL], b01[QPL], b10[QPL], b11[QPL];
#pragma unroll
  for (int i = 0; i < QPL; ++i) {
    if (em.q[i] & (1 << 13)) {
      const int o = em.q[i] & 0x7ff;
      const T2 v0 = *reinterpret_cast<const T2*>(Bc + o);
      const T2 v1 = *reinterpret_cast<const T2*>(Bc + o + W2);
      const bool sw = (em.q[i] >> 11) & 1;
      b00[i] = sw ? v0.y : v0.x;
      b01[i] = sw ? v0.x : v0.y;
      b10[i] = sw ? v1.y : v1.x;
      b11[i] = sw ? v1.x : v1.y;
    }
  }
  const bool any = __any_sync(0xffffffffu, rot);
  if (!any) {
    PHASE_COUNT(8);  // profiling builds: rotation-free EVD steps
#pragma unroll
    for (int i = 0; i < QPL; ++i) {
      if (em.q[i] & (1 << 13)) {
        Bn[em.st[i][0] & 0xffff] = b00[i];
        Bn[em.st[i][0] >> 16] = b01[i];
        Bn[em.st[i][1] & 0xffff] = b10[i];
        Bn[em.st[i][1] >> 16] = b11[i];
      }
    }
#pragma unroll
    for (int k = 0; k < W2; ++k) y[rr_dest(k, W2)] = x[k];
    return false;
  }
  __syncwarp();
#pragma unroll
  for (int i = 0; i < QPL; ++i) {
    if (em.q[i] & (1 << 13)) {
      const T2 gp = cs[(em.q[i] >> 16) & (NPR - 1)];
      const bool own_lo = (em.q[i] >> 12) & 1;
      const T rc = own_lo ? c : gp.x, rs = own_lo ? s : gp.y;  // rotation of the row pair
      const T cc = own_lo ? gp.x : c, cs_ = own_lo ? gp.y : s;  // rotation of the column pair
      // columns (2hi, 2hi+1): B G_hi
      const T c0 = fma(cs_, b01[i], cc * b00[i]), c1 = fma(-cs_, b00[i], cc * b01[i]);
      const T d0 = fma(cs_, b11[i], cc * b10[i]), d1 = fma(-cs_, b10[i], cc * b11[i]);
      // rows (2lo, 2lo+1): G_lo^T (B G_hi)
      Bn[em.st[i][0] & 0xffff] = fma(rs, d0, rc * c0);
      Bn[em.st[i][0] >> 16] = fma(rs, d1, rc * c1);
      Bn[em.st[i][1] & 0xffff] = fma(-rs, c0, rc * d0);
      Bn[em.st[i][1] >> 16] = fma(-rs, c1, rc * d1);
    }
  }
  // J <- J G in slot order; outputs move to their next slots (register rename).
#pragma unroll
  for (int k = 0; k < NPR; ++k) {
    const T2 g = cs[k];
    const T a = x[2 * k], b = x[2 * k + 1];
    y[rr_dest(2 * k, W2)] = fma(g.y, b, g.x * a);
    y[rr_dest(2 * k + 1, W2)] = fma(-g.y, a, g.x * b);
  }
  return true;
}

// ---- Inner EVD step, full-symmetric layout (default, WCSVD_EVD_FULL = 1) ----
// B is stored as the FULL symmetric 2w x 2w matrix in slot order (row stride 2w, both triangles). Lane
// L works for pair k = L mod w (its own rotation) and owns the quads B(k, l), l = k + d (mod w), for its
// share of d: with both triangles stored, the quad is always loaded as rows (2k, 2k+1) x columns
// (2l, 2l+1) -- lane-uniform shape, no swaps and no "which side am I" selects -- rotated by the lane's
// own (c, s) on the rows and the partner's (c, s) (one shuffle from lane l) on the columns, and written
// with its transpose to the slots both index pairs move to. A quarter-warp's eight LDS.128 hit eight
// distinct 16-byte bank groups (group = (k + d) mod 8), so no swizzle is needed.
template <int W2>
struct EvdMapF {
  static constexpr int NPR = W2 / 2, LPP = 32 / NPR, HALF = NPR / 2;
  static constexpr int QPL = (HALF + LPP - 1) / LPP;
  int ld[QPL];      // bits 0-11 load offset of B(2k, 2l); bits 12-16 partner l; bit 17 valid
  int st[QPL][4];   // store offsets (16-bit pairs) of the quad and of its transpose
  int dld, dst[2];  // diagonal block load offset (2k, 2k); stores (moved slots): (p,p) | (q,q) << 16, (p,q) | (q,p) << 16
  __device__ __forceinline__ void init(int lane) {
    const int k = lane & (NPR - 1), h = lane / NPR;
    const int k0 = rr_dest(2 * k, W2), k1 = rr_dest(2 * k + 1, W2);
#pragma unroll
    for (int i = 0; i < QPL; ++i) {
      const int d = 1 + h * QPL + i;
      const bool valid = d < HALF || (d == HALF && k < HALF);
      const int l = (k + d) & (NPR - 1);
      const int l0 = rr_dest(2 * l, W2), l1 = rr_dest(2 * l + 1, W2);
      ld[i] = valid ? ((2 * k) * W2 + 2 * l) | (l << 12) | (1 << 17) : 0;
      st[i][0] = (k0 * W2 + l0) | ((k0 * W2 + l1) << 16);
      st[i][1] = (k1 * W2 + l0) | ((k1 * W2 + l1) << 16);
      st[i][2] = (l0 * W2 + k0) | ((l1 * W2 + k0) << 16);  // transpose: B'(l, k) = B'(k, l)^T
      st[i][3] = (l0 * W2 + k1) | ((l1 * W2 + k1) << 16);
    }
    dld = (2 * k) * W2 + 2 * k;
    dst[0] = (k0 * W2 + k0) | ((k1 * W2 + k1) << 16);
    dst[1] = (k0 * W2 + k1) | ((k1 * W2 + k0) << 16);
  }
};

template <int W2>
__device__ __forceinline__ bool evd_step_full(const double* __restrict__ Bc, double* __restrict__ Bn, double2* cs,
                                              const EvdMapF<W2>& em, int lane, double tol2, double (&x)[W2]) {
  constexpr int NPR = W2 / 2, QPL = EvdMapF<W2>::QPL;
  const double2 dv0 = *reinterpret_cast<const double2*>(Bc + em.dld);       // b_pp, b_pq
  const double bqq = Bc[em.dld + W2 + 1];
  double c, s;
#if WCSVD_EVD_ROT32
  const bool rot = jacobi_rotation_f32(dv0.x, bqq, dv0.y, tol2, c, s);
#else
  double t;
  const bool rot = jacobi_rotation(dv0.x, bqq, dv0.y, tol2, c, s, t);
#endif
  double b00[QPL], b01[QPL], b10[QPL], b11[QPL];
#pragma unroll
  for (int i = 0; i < QPL; ++i) {
    if (em.ld[i] & (1 << 17)) {
      const int o = em.ld[i] & 0xfff;
      const double2 v0 = *reinterpret_cast<const double2*>(Bc + o);
      const double2 v1 = *reinterpret_cast<const double2*>(Bc + o + W2);
      b00[i] = v0.x; b01[i] = v0.y; b10[i] = v1.x; b11[i] = v1.y;
    }
  }
  if (lane < NPR) {
    cs[lane] = make_double2(c, s);
#if WCSVD_EVD_ROT32
    // general two-sided update of the diagonal block (the fp32 angle leaves b_pq' ~ 1e-7 b_pq, kept)
    const double c0 = fma(s, dv0.y, c * dv0.x), c1 = fma(-s, dv0.x, c * dv0.y);
    const double d0 = fma(s, bqq, c * dv0.y), d1 = fma(-s, dv0.y, c * bqq);
    const double pp = rot ? fma(s, d0, c * c0) : dv0.x, qq = rot ? fma(-s, c1, c * d1) : bqq;
    const double pq = rot ? fma(s, d1, c * c1) : dv0.y;
#else
    const double pp = rot ? fma(t, dv0.y, dv0.x) : dv0.x, qq = rot ? fma(-t, dv0.y, bqq) : bqq;
    const double pq = rot ? 0.0 : dv0.y;
#endif
    Bn[em.dst[0] & 0xffff] = pp;
    Bn[em.dst[0] >> 16] = qq;
    Bn[em.dst[1] & 0xffff] = pq;
    Bn[em.dst[1] >> 16] = pq;
  }
  const bool any = __any_sync(0xffffffffu, rot);
#pragma unroll
  for (int i = 0; i < QPL; ++i) {
    const int l = (em.ld[i] >> 12) & 31;
    const double cl = __shfl_sync(0xffffffffu, c, l), sl = __shfl_sync(0xffffffffu, s, l);
    if (em.ld[i] & (1 << 17)) {
      // columns (2l, 2l+1): B G_l; rows (2k, 2k+1): G_k^T (B G_l)
      const double c0 = fma(sl, b01[i], cl * b00[i]), c1 = fma(-sl, b00[i], cl * b01[i]);
      const double d0 = fma(sl, b11[i], cl * b10[i]), d1 = fma(-sl, b10[i], cl * b11[i]);
      const double n00 = fma(s, d0, c * c0), n01 = fma(s, d1, c * c1);
      const double n10 = fma(-s, c0, c * d0), n11 = fma(-s, c1, c * d1);
      Bn[em.st[i][0] & 0xffff] = n00;
      Bn[em.st[i][0] >> 16] = n01;
      Bn[em.st[i][1] & 0xffff] = n10;
      Bn[em.st[i][1] >> 16] = n11;
      Bn[em.st[i][2] & 0xffff] = n00;  // (l0, k0)
      Bn[em.st[i][2] >> 16] = n01;     // (l1, k0)
      Bn[em.st[i][3] & 0xffff] = n10;  // (l0, k1)
      Bn[em.st[i][3] >> 16] = n11;     // (l1, k1)
    }
  }
  if (any) __syncwarp();
  // J <- J G in slot order, IN PLACE: every output goes straight into the register of the slot it
  // moves to (common.cuh ring). Pairs are visited from the last to the first: the top output of
  // pair k lands in top[k+1] (pair k+1 was already read), the bottom output is held one pair
  // (`pend`) until pair k-1 has read bot[k-1]. One register set instead of the x -> y ping-pong
  // (-64 registers); the same operations on the same operands, so the bits are unchanged.
  double pend = 0.0;
#pragma unroll
  for (int k = NPR - 1; k >= 0; --k) {
    const double a = x[2 * k], b = x[2 * k + 1];
    if (k < NPR - 1) x[2 * k + 1] = pend;
    double na = a, nb = b;
    if (any) {
      const double2 g = cs[k];
      na = fma(g.y, b, g.x * a);
      nb = fma(-g.y, a, g.x * b);
    }
    x[rr_dest(2 * k, W2)] = na;
    if (k >= 1) pend = nb;
    else x[rr_dest(1, W2)] = nb;
  }
  return any;
}

// ---- Group (i) inner solve, PANEL path (Alg 2 l.8-9; Step 2 group (i), PAPER.md:175;
// DESIGN.md §5.2c): J from the SVD of the pair panel P = [A_i A_j] itself, by one-sided Jacobi. The M x 2w
// panel does not fit one warp's registers, so it is first compressed to its 2w x 2w triangular factor R
// (P = Q R, Q orthonormal; R from the Cholesky factorisation of the Gram B = P^T P = R^T R -- CholeskyQR):
// one-sided Jacobi on the columns of R produces exactly the rotations of one-sided Jacobi on the
// columns of P (same alpha = ||p_i||^2, beta, gamma = p_i^T p_j), eq (3)-(4) PAPER.md:76-81. Cholesky:
// lane c holds row / column c of B, pivots broadcast by shuffle, the trailing update reads row j of R
// from a shared row buffer; R is then transposed so that lane r holds row r of R. Per step: 16 products, a
// fixed-order butterfly reduce-scatter of the 16 dot products (lane L ends with pair L/2's gamma),
// eq (4) in the pair's two lanes, eq (6) norm updates, the (c, s) of the step logged
// to shared memory, and the 16 column rotations of the lane's row with register renaming. J is built
// afterwards from the log. Falls back to the two-sided sweep when a Cholesky pivot falls below
// 2^-24 of its column's norm^2 (nearly dependent columns: R would lose relative accuracy).
constexpr double kCholTau = 5.9604644775390625e-08;  // 2^-24

// One one-sided step: x = row `lane` of R (slot order) -> y (moved slots); alpha = ||column lane||^2.
__device__ __forceinline__ bool onesided_step(const double (&x)[32], double (&y)[32], double& alpha,
                                              double2* __restrict__ logs, int lane, double tol2) {
  double v[16];
#pragma unroll
  for (int k = 0; k < 16; ++k) v[k] = x[2 * k] * x[2 * k + 1];
  // butterfly reduce-scatter: level o keeps the half selected by lane bit log2(o), lane L -> pair L/2
#pragma unroll
  for (int o = 16, n = 8; o >= 2; o >>= 1, n >>= 1) {
    const bool up = (lane & o) != 0;
#pragma unroll
    for (int i = 0; i < n; ++i) {
      const double keep = up ? v[n + i] : v[i];
      const double send = up ? v[i] : v[n + i];
      v[i] = keep + __shfl_xor_sync(0xffffffffu, send, o);
    }
  }
  const double g = v[0] + __shfl_xor_sync(0xffffffffu, v[0], 1);  // gamma_{lane/2}, bitwise equal in both lanes
  const double ao = __shfl_xor_sync(0xffffffffu, alpha, 1);
  const bool odd = lane & 1;
  const double ap = odd ? ao : alpha, aq = odd ? alpha : ao;  // (alpha_2k, alpha_2k+1) in both lanes
  double c, s, t;
  const bool rot = jacobi_rotation(ap, aq, g, tol2, c, s, t);
  if (rot) alpha = odd ? fma(-t, g, alpha) : fma(t, g, alpha);  // eq (6)
  if (!odd) logs[lane >> 1] = make_double2(c, s);
  alpha = __shfl_sync(0xffffffffu, alpha, rr_src(lane, 32));  // norms move with their columns
  const bool any = __any_sync(0xffffffffu, rot);
  __syncwarp();
#pragma unroll
  for (int k = 0; k < 16; ++k) {
    const double2 q = logs[k];
    const double a = x[2 * k], b = x[2 * k + 1];
    y[rr_dest(2 * k, 32)] = fma(q.y, b, q.x * a);
    y[rr_dest(2 * k + 1, 32)] = fma(-q.y, a, q.x * b);
  }
  return any;
}

// J <- J G of logged step `st` (or the rename only when the step did not rotate).
__device__ __forceinline__ void jbuild_step(const double (&x)[32], double (&y)[32], const double2* logs, bool any) {
  if (!any) {
#pragma unroll
    for (int k = 0; k < 32; ++k) y[rr_dest(k, 32)] = x[k];
    return;
  }
#pragma unroll
  for (int k = 0; k < 16; ++k) {
    const double2 q = logs[k];
    const double a = x[2 * k], b = x[2 * k + 1];
    y[rr_dest(2 * k, 32)] = fma(q.y, b, q.x * a);
    y[rr_dest(2 * k + 1, 32)] = fma(-q.y, a, q.x * b);
  }
}

// Returns false (nothing changed) if the Cholesky route does not apply; else ja = J (row `lane`,
// slot = original order) and *rotated.
__device__ __forceinline__ bool evd_fast32(const double* __restrict__ B0, double* __restrict__ scratch, int lane,
                                        double tol2, double (&ja)[32], bool* rotated) {
  // scratch: >= 1056 doubles (transpose 32 x 33; the Cholesky row buffers and the (c, s) log alias it)
  double b[32], r[32];
#pragma unroll
#if WCSVD_EVD_FULL
  for (int c = 0; c < 32; ++c) b[c] = B0[lane * 32 + c];
  const double dl = B0[lane * 33];  // ||column lane||^2 (original)
#else
  for (int c = 0; c < 32; ++c) b[c] = B0[evd_phys_sym<32>(lane, c)];
  const double dl = B0[evd_phys<32>(lane, lane)];
#endif
  bool ok = true;
#pragma unroll
  for (int j = 0; j < 32; ++j) {
    const double d = __shfl_sync(0xffffffffu, b[j], j);
    const double d0 = __shfl_sync(0xffffffffu, dl, j);
    ok &= !(d0 > 0.0) || d > kCholTau * d0;
    const double inv = (d0 > 0.0 && d > 0.0) ? rsqrt(d) : 0.0;
    const double rj = (lane >= j) ? b[j] * inv : 0.0;  // R[j][lane]
    r[j] = rj;
    double* rb = scratch + 32 * (j & 1);
    rb[lane] = rj;
    __syncwarp();
#pragma unroll
    for (int c = j + 1; c < 32; ++c) b[c] = fma(-rj, rb[c], b[c]);
  }
  if (!ok) return false;  // warp-uniform (every lane saw every pivot)
  __syncwarp();
  // transpose: lane c holds column c of R (r[j] = R[j][c]); lane r needs row r
#pragma unroll
  for (int j = 0; j < 32; ++j) scratch[j * 33 + lane] = r[j];
  __syncwarp();
#pragma unroll
  for (int c = 0; c < 32; ++c) b[c] = scratch[lane * 33 + c];
  __syncwarp();
  double alpha = dl;
  double2* logs = reinterpret_cast<double2*>(scratch);  // [31][16]
  unsigned mask = 0;
  // 31 steps (odd): x->y first, then pairs y->x, x->y; slots return to the original order
  mask |= (unsigned)onesided_step(b, r, alpha, logs, lane, tol2);
#pragma unroll 1
  for (int st = 1; st < 31; st += 2) {
    mask |= (unsigned)onesided_step(r, b, alpha, logs + 16 * st, lane, tol2) << st;
    mask |= (unsigned)onesided_step(b, r, alpha, logs + 16 * (st + 1), lane, tol2) << (st + 1);
  }
  *rotated = mask != 0;
  if (!mask) return true;
  // J = product of the logged step rotations (slot order, rows in lanes)
#pragma unroll
  for (int s = 0; s < 32; ++s) b[s] = (lane == s) ? 1.0 : 0.0;
  jbuild_step(b, r, logs, mask & 1u);
#pragma unroll 1
  for (int st = 1; st < 31; st += 2) {
    jbuild_step(r, b, logs + 16 * st, (mask >> st) & 1u);
    jbuild_step(b, r, logs + 16 * (st + 1), (mask >> (st + 1)) & 1u);
  }
#pragma unroll
  for (int s = 0; s < 32; ++s) ja[s] = r[s];
  return true;
}

// Process one column-block pair (I, J) of the working matrix with one warp. Returns true if it
// rotated (A and V panels updated); counts inner sweeps into *inner.
template <int W2, bool PANEL = false>
__device__ bool process_pair(const WarpSmem<W2>& ws, const EvdMap<W2>* s_em, double* Wm, int ld, int mrows,
                             double* Vm, int ldv, int vrows, int I, int J, double tol2, int inner_cap,
                             int lane, int* inner) {
  using C = PairCfg<W2>;
  constexpr int CG = C::CG, BS = C::BS;
  PHASE_T0();
  // (1) Gram B = P^T P, P = [W_I W_J] (Alg 1 l.5), upper triangle into the EVD layout.
  double* B0 = ws.B;
  double* B1 = ws.B + W2 * W2;
  {
    double acc[C::NTU][2];
    gram_tiles_async<W2, WarpSmem<W2>::NSTAGE>(ws.ring, Wm, ld, mrows, I, J, lane, acc);
    int t = 0;
#pragma unroll
    for (int a = 0; a < CG; ++a)
#pragma unroll
      for (int b = a; b < CG; ++b, ++t)
#pragma unroll
        for (int e = 0; e < 2; ++e) {
          const int row = 8 * a + (lane >> 2), col = 8 * b + 2 * (lane & 3) + e;
#if WCSVD_EVD_FULL
          B0[row * W2 + col] = acc[t][e];
          if (a != b) B0[col * W2 + row] = acc[t][e];
#else
          if (a != b || row <= col) B0[evd_phys<W2>(row, col)] = acc[t][e];
#endif
        }
  }
  __syncwarp();
  PHASE_MARK(0);
  // (4) off-norm test on the Gram (Z6): skip the pair if every b_pq^2 <= tol^2 b_pp b_qq.
  bool need = false;
  bool pert_ok = true;  // R-PERT: every rotating b_pq is small against its diagonal gap
  {
#if WCSVD_EVD_FULL
#define BIDX(a, b) ((a) * W2 + (b))
#else
#define BIDX(a, b) evd_phys<W2>(a, b)
#endif
    const double bqq = (lane < W2) ? B0[BIDX(lane, lane)] : 0.0;
#pragma unroll 4
    for (int p = 0; p < W2 - 1; ++p) {
      const double bpp = B0[BIDX(p, p)];  // broadcast
      const double bpq = (lane < W2 && lane > p) ? B0[BIDX(p, lane)] : 0.0;
#undef BIDX
      const double ab = bpp * bqq;
      const bool rot = (lane > p && ab > 0.0 && bpq * bpq > tol2 * ab);
      need |= rot;
      pert_ok &= !rot || fabs(bpq) <= kPertDelta * fabs(bpp - bqq);
    }
  }
  PHASE_MARK(1);
  PHASE_COUNT(7);
  if (!__any_sync(0xffffffffu, need)) return false;
#ifdef WCSVD_PHASE_PROFILE
  {  // how close to diagonal is B? max over rotating pairs of |b_pq| / |b_pp - b_qq| (experiment)
    double mx = 0.0;
    if (lane < W2) {
      const double bqq = B0[lane * W2 + lane];
      for (int p = 0; p < lane; ++p) {
        const double bpp = B0[p * W2 + p], bpq = B0[p * W2 + lane];
        if (bpq * bpq > tol2 * bpp * bqq) mx = fmax(mx, fabs(bpq) / fabs(bpp - bqq));
      }
    }
    for (int o = 16; o > 0; o >>= 1) mx = fmax(mx, __shfl_xor_sync(0xffffffffu, mx, o));
    if (mx <= 1e-2) PHASE_COUNT(10);
    if (mx <= 2e-3) PHASE_COUNT(9);
    if (mx <= 1e-4) PHASE_COUNT(11);
  }
#endif
  // (2) EVD of B (Alg 1 l.6): threshold parallel Jacobi, B and J in slot order.
  double ja[W2], jb[W2];
  bool rotated = false;
  int isw = 0;
  bool panel_done = false;
  const bool pert = WCSVD_L1_PERT && WCSVD_EVD_FULL && !PANEL && __all_sync(0xffffffffu, pert_ok);
  if (pert) {
    // R-PERT: lane p builds row p of J = I + E, E_pq = b_pq / (b_qq - b_pp) for the rotating pairs
    // (the first-order eigenvectors of a nearly diagonal B; antisymmetric)
    const double bpp = (lane < W2) ? B0[lane * W2 + lane] : 1.0;
#pragma unroll
    for (int q = 0; q < W2; ++q) {
      const double bqq = B0[q * W2 + q];  // broadcast
      const double bpq = (lane < W2) ? B0[lane * W2 + q] : 0.0;
      const double ab = bpp * bqq;
      const bool rot = q != lane && ab > 0.0 && bpq * bpq > tol2 * ab;
      ja[q] = (q == lane) ? 1.0 : (rot ? bpq / (bqq - bpp) : 0.0);
    }
    rotated = true;
    isw = 1;
    panel_done = true;
  }
  if constexpr (PANEL && W2 == 32) {
    // group (i): one-sided Jacobi of the (CholeskyQR-compressed) panel; group (ii) below if a pivot is tiny
    if (inner_cap == 1) panel_done = evd_fast32(B0, B1, lane, tol2, ja, &rotated);
    if (panel_done) isw = 1;
  }
  if (!panel_done) {
#if WCSVD_EVD_FULL
  EvdMapF<W2> em;  // lane-static map, rebuilt per pair (no registers held outside the EVD)
#define EVD_STEP evd_step_full<W2>
#else
  EvdMap<W2> em;
#define EVD_STEP evd_step<W2>
#endif
  em.init(lane);
#pragma unroll
  for (int s = 0; s < W2; ++s) ja[s] = (lane == s) ? 1.0 : 0.0;
  for (; isw < inner_cap; ++isw) {
#if WCSVD_EVD_FULL
    // W2-1 steps (odd): B ping-pongs B0 -> B1 -> B0 ..., ends in B1; J is updated in place in ja and
    // its slots are back in order after the sweep.
    bool any = EVD_STEP(B0, B1, ws.cs, em, lane, tol2, ja);
    __syncwarp();
    for (int r = 1; r < W2 - 1; r += 2) {
      any |= EVD_STEP(B1, B0, ws.cs, em, lane, tol2, ja);
      __syncwarp();
      any |= EVD_STEP(B0, B1, ws.cs, em, lane, tol2, ja);
      __syncwarp();
    }
#else
    // W2-1 steps (odd): x->y first, then pairs y->x, x->y; ends in jb / B1, slots back in order.
    bool any = EVD_STEP(B0, B1, ws.cs, em, lane, tol2, ja, jb);
    __syncwarp();
    for (int r = 1; r < W2 - 1; r += 2) {
      any |= EVD_STEP(B1, B0, ws.cs, em, lane, tol2, jb, ja);
      __syncwarp();
      any |= EVD_STEP(B0, B1, ws.cs, em, lane, tol2, ja, jb);
      __syncwarp();
    }
#pragma unroll
    for (int s = 0; s < W2; ++s) ja[s] = jb[s];
#endif
#undef EVD_STEP
    double* tmp = B0;
    B0 = B1;
    B1 = tmp;
    rotated |= any;
    if (!any) break;
  }
  }
  *inner += pert ? 1 : isw + (isw < inner_cap ? 1 : 0);
  PHASE_MARK(2);
  PHASE_COUNT(6);
  if (!rotated) return false;
  // Stage J; Newton-Schulz (Z9(ii)): E = J^T J - I, J' = J - J E / 2.
  if (lane < W2) {
#pragma unroll
    for (int s = 0; s < W2; ++s) ws.S[lane * BS + s] = ja[s];
  }
  __syncwarp();
#if WCSVD_L1_NS
  for (int nsp = 0; nsp < (pert ? kPertNS : 1); ++nsp) {
  if (nsp) {  // R-PERT: a second Newton-Schulz step on J' (J = I + E is orthogonal only to O(E^2))
    if (lane < W2) {
#pragma unroll
      for (int s = 0; s < W2; ++s) ws.S[lane * BS + s] = ws.B[lane * BS + s];
    }
    __syncwarp();
  }
  {
    const double* ptr[CG];
#pragma unroll
    for (int c = 0; c < CG; ++c) ptr[c] = ws.S + (lane & 3) * BS + 8 * c + (lane >> 2);
    double acc[C::NTU][2];
    gram_tiles<W2>(ptr, W2, BS, acc);
    __syncwarp();
    store_sym<W2>(ws.B, acc, lane, 1.0);
  }
  __syncwarp();
  double jn[CG][CG][2];
#pragma unroll
  for (int i = 0; i < CG; ++i)
#pragma unroll
    for (int j = 0; j < CG; ++j) {
      double acc[2] = {0.0, 0.0};
#pragma unroll
      for (int kk = 0; kk < W2 / 4; ++kk)
        dmma884(acc, ws.S[(8 * i + (lane >> 2)) * BS + 4 * kk + (lane & 3)],
                ws.B[(4 * kk + (lane & 3)) * BS + 8 * j + (lane >> 2)]);
#pragma unroll
      for (int e = 0; e < 2; ++e)
        jn[i][j][e] = fma(-0.5, acc[e], ws.S[(8 * i + (lane >> 2)) * BS + 8 * j + 2 * (lane & 3) + e]);
    }
  __syncwarp();
#pragma unroll
  for (int i = 0; i < CG; ++i)
#pragma unroll
    for (int j = 0; j < CG; ++j)
#pragma unroll
      for (int e = 0; e < 2; ++e) ws.B[(8 * i + (lane >> 2)) * BS + 8 * j + 2 * (lane & 3) + e] = jn[i][j][e];
  __syncwarp();
  }
  const double* jsrc = ws.B;
#else
  const double* jsrc = ws.S;  // ablation build (-DWCSVD_L1_NS=0): J applied without the cleanup step
#endif
  double jf[W2 / 4][CG];
#pragma unroll
  for (int kk = 0; kk < W2 / 4; ++kk)
#pragma unroll
    for (int nb = 0; nb < CG; ++nb) jf[kk][nb] = jsrc[(4 * kk + (lane & 3)) * BS + 8 * nb + (lane >> 2)];
  PHASE_MARK(3);
  // (3) A_ij <- A_ij J (Alg 1 l.7) and V_ij <- V_ij J.
  __syncwarp();  // the ring aliases B: every lane holds its J' fragments before slabs land
  apply_rotation_async<W2, WarpSmem<W2>::NSTAGE, 1>(ws.ring, Wm, ld, mrows, I, J, lane, jf);
  PHASE_MARK(4);
  apply_rotation_async<W2, WarpSmem<W2>::NSTAGE, 2>(ws.ring, Vm, ldv, vrows, I, J, lane, jf);
  PHASE_MARK(5);
  return true;
}
// ---- fp32 Gram path (wcsvd_batched_f32): the same pair steps in single precision ----
// sm_100a has no full-precision fp32 MMA (DMMA is fp64 only, TF32 keeps 10 mantissa bits), so the two
// contractions run on the FFMA pipe: lane l owns column l of the Gram / of the updated panel (two lanes
// per column when 2w = 16, one per 8-row half of a slab, summed in fixed order), panel slabs arrive
// through the same per-warp cp.async ring (16 rows x 2w columns, 80-byte column stride), every value a
// lane needs from another column is a broadcast LDS.128 of 4 consecutive rows. The EVD is evd_step<W2,
// float>, the Newton-Schulz cleanup is two 2w^3 FFMA contractions in shared memory. The working copy
// W, V is fp32 (half the bytes of the fp64 path).
template <int W2>
struct WarpSmemF {
  float* B;    // EVD ping-pong (2 x W2 x W2, slot layout); afterwards E = J^T J - I ([W2][BS])
  float* S;    // [W2][BS] staged J
  float2* cs;  // [W2 / 2]
  float* ring; // [NSTAGE][W2][SLF]
  static constexpr int BS = W2 + 1;
  static constexpr int SLF = 20;  // ring column stride (floats): 16 rows + 4 pad, 16-byte chunks
  static constexpr int NSTAGE = WCSVD_L1_NSTAGE;
  static constexpr int SLAB = W2 * SLF;
  __host__ __device__ static constexpr size_t region() {
    return (2 * W2 * BS > NSTAGE * SLAB ? 2 * W2 * BS : NSTAGE * SLAB) * sizeof(float);
  }
  __host__ __device__ static constexpr size_t bytes() { return region() + sizeof(float2) * (W2 / 2); }
};

// chunk i of this lane: column (lane + 32 i) / 4, rows 4 ((lane + 32 i) % 4) .. +3 of the slab
template <int W2>
__device__ __forceinline__ void slab_issue_f(float* ring, const float* base, const int (&coff)[W2 / 8], int r0,
                                             int st, int lane) {
  float* dst = ring + st * WarpSmemF<W2>::SLAB;
#pragma unroll
  for (int i = 0; i < W2 / 8; ++i) {
    const int q = lane + 32 * i, c = q >> 2, h = q & 3;
    cp_async16(dst + c * WarpSmemF<W2>::SLF + 4 * h, base + coff[i] + r0 + 4 * h);
  }
}

template <int W2>
__device__ __forceinline__ void slab_offsets_f(int (&coff)[W2 / 8], int I, int J, int ld, int lane) {
#pragma unroll
  for (int i = 0; i < W2 / 8; ++i) coff[i] = pcol<W2>((lane + 32 * i) >> 2, I, J) * ld;
}

// acc[i] = sum_r P[r][i] P[r][col] over the panel rows (this lane's half of every slab), then the two
// halves are combined (2w = 16): B[i][col] for every i, lane = (half, col).
template <int W2>
__device__ __forceinline__ void gram_f32(float* ring, const float* base, int ld, int rows, int I, int J, int lane,
                                         float (&acc)[W2]) {
  constexpr int SLF = WarpSmemF<W2>::SLF, NS = WarpSmemF<W2>::NSTAGE, LPC = 32 / W2, RPL = 16 / LPC;
  const int col = lane % W2, half = lane / W2;
#pragma unroll
  for (int i = 0; i < W2; ++i) acc[i] = 0.0f;
  int coff[W2 / 8];
  slab_offsets_f<W2>(coff, I, J, ld, lane);
  const int nslab = rows >> 4;
#pragma unroll
  for (int j = 0; j < NS - 1; ++j) {
    if (j < nslab) slab_issue_f<W2>(ring, base, coff, 16 * j, j, lane);
    cp_async_commit();
  }
  for (int sl = 0; sl < nslab; ++sl) {
    if (sl + NS - 1 < nslab) slab_issue_f<W2>(ring, base, coff, 16 * (sl + NS - 1), (sl + NS - 1) % NS, lane);
    cp_async_commit();
    cp_async_wait<NS - 1>();
    __syncwarp();
    const float* st = ring + (sl % NS) * WarpSmemF<W2>::SLAB;
#pragma unroll
    for (int r4 = 0; r4 < RPL; r4 += 4) {
      const float4 own = *reinterpret_cast<const float4*>(st + col * SLF + half * RPL + r4);
#pragma unroll
      for (int i = 0; i < W2; ++i) {
        const float4 v = *reinterpret_cast<const float4*>(st + i * SLF + half * RPL + r4);
        acc[i] = fmaf(v.x, own.x, acc[i]);
        acc[i] = fmaf(v.y, own.y, acc[i]);
        acc[i] = fmaf(v.z, own.z, acc[i]);
        acc[i] = fmaf(v.w, own.w, acc[i]);
      }
    }
    __syncwarp();
  }
  if constexpr (LPC == 2) {
#pragma unroll
    for (int i = 0; i < W2; ++i) acc[i] += __shfl_xor_sync(0xffffffffu, acc[i], 16);  // commutative: same bits
  }
}

// X <- X J' for the panel of pair (I, J): lane (half, col) computes column col of its rows of every
// slab from jc[k] = J'[k][col]; results stored in place (a slab's rows are read before overwritten).
template <int W2>
__device__ __forceinline__ void apply_f32(float* ring, float* base, int ld, int rows, int I, int J, int lane,
                                          const float (&jc)[W2]) {
  constexpr int SLF = WarpSmemF<W2>::SLF, NS = WarpSmemF<W2>::NSTAGE, LPC = 32 / W2, RPL = 16 / LPC;
  const int col = lane % W2, half = lane / W2;
  int coff[W2 / 8];
  slab_offsets_f<W2>(coff, I, J, ld, lane);
  float* out = base + (size_t)pcol<W2>(col, I, J) * ld + half * RPL;
  const int nslab = rows >> 4;
#pragma unroll
  for (int j = 0; j < NS - 1; ++j) {
    if (j < nslab) slab_issue_f<W2>(ring, base, coff, 16 * j, j, lane);
    cp_async_commit();
  }
  for (int sl = 0; sl < nslab; ++sl) {
    if (sl + NS - 1 < nslab) slab_issue_f<W2>(ring, base, coff, 16 * (sl + NS - 1), (sl + NS - 1) % NS, lane);
    cp_async_commit();
    cp_async_wait<NS - 1>();
    __syncwarp();
    const float* st = ring + (sl % NS) * WarpSmemF<W2>::SLAB;
#pragma unroll
    for (int r4 = 0; r4 < RPL; r4 += 4) {
      float4 o = make_float4(0.f, 0.f, 0.f, 0.f);
#pragma unroll
      for (int k = 0; k < W2; ++k) {
        const float4 v = *reinterpret_cast<const float4*>(st + k * SLF + half * RPL + r4);
        o.x = fmaf(v.x, jc[k], o.x);
        o.y = fmaf(v.y, jc[k], o.y);
        o.z = fmaf(v.z, jc[k], o.z);
        o.w = fmaf(v.w, jc[k], o.w);
      }
      __stcg(reinterpret_cast<float4*>(out + 16 * sl + r4), o);
    }
    __syncwarp();
  }
}

template <int W2>
__device__ bool process_pair_f32(const WarpSmemF<W2>& ws, float* Wm, int ld, int mrows, float* Vm, int ldv,
                                 int vrows, int I, int J, float tol2, int inner_cap, int lane, int* inner) {
  constexpr int BS = WarpSmemF<W2>::BS;
  const int col = lane % W2;
  float* B0 = ws.B;
  float* B1 = ws.B + W2 * W2;
  // (1) Gram (Alg 1 l.5), upper triangle into the EVD layout
  {
    float acc[W2];
    gram_f32<W2>(ws.ring, Wm, ld, mrows, I, J, lane, acc);
    __syncwarp();  // the ring aliases B
    if (lane < W2) {
#pragma unroll
      for (int i = 0; i < W2; ++i)
        if (i <= col) B0[evd_phys<W2>(i, col)] = acc[i];
    }
  }
  __syncwarp();
  // (4) off-norm test (Z6)
  bool need = false;
  {
    const float bqq = (lane < W2) ? B0[evd_phys<W2>(lane, lane)] : 0.0f;
#pragma unroll 4
    for (int p = 0; p < W2 - 1; ++p) {
      const float bpp = B0[evd_phys<W2>(p, p)];
      const float bpq = (lane < W2 && lane > p) ? B0[evd_phys<W2>(p, lane)] : 0.0f;
      const float ab = bpp * bqq;
      need |= (lane > p && ab > 0.0f && bpq * bpq > tol2 * ab);
    }
  }
  if (!__any_sync(0xffffffffu, need)) return false;
  // (2) EVD (Alg 1 l.6), threshold parallel Jacobi in fp32
  EvdMap<W2> em;
  em.init(lane);
  float ja[W2], jb[W2];
#pragma unroll
  for (int s = 0; s < W2; ++s) ja[s] = (lane == s) ? 1.0f : 0.0f;
  bool rotated = false;
  int isw = 0;
  for (; isw < inner_cap; ++isw) {
    bool any = evd_step<W2, float>(B0, B1, ws.cs, em, lane, tol2, ja, jb);
    __syncwarp();
    for (int r = 1; r < W2 - 1; r += 2) {
      any |= evd_step<W2, float>(B1, B0, ws.cs, em, lane, tol2, jb, ja);
      __syncwarp();
      any |= evd_step<W2, float>(B0, B1, ws.cs, em, lane, tol2, ja, jb);
      __syncwarp();
    }
#pragma unroll
    for (int s = 0; s < W2; ++s) ja[s] = jb[s];
    float* tmp = B0;
    B0 = B1;
    B1 = tmp;
    rotated |= any;
    if (!any) break;
  }
  *inner += isw + (isw < inner_cap ? 1 : 0);
  if (!rotated) return false;
  // Stage J (row lane), Newton-Schulz (Z9(ii)): E = J^T J - I, J' = J - J E / 2; lane keeps column col of J'.
  if (lane < W2) {
#pragma unroll
    for (int s = 0; s < W2; ++s) ws.S[lane * BS + s] = ja[s];
  }
  __syncwarp();
  float jc[W2];
  {
    float e[W2];
#pragma unroll
    for (int i = 0; i < W2; ++i) e[i] = 0.0f;
#pragma unroll 4
    for (int k = 0; k < W2; ++k) {
      const float jk = ws.S[k * BS + col];
#pragma unroll
      for (int i = 0; i < W2; ++i) e[i] = fmaf(ws.S[k * BS + i], jk, e[i]);
    }
    __syncwarp();
    if (lane < W2) {
#pragma unroll
      for (int i = 0; i < W2; ++i) ws.B[i * BS + col] = e[i] - (i == col ? 1.0f : 0.0f);
    }
    __syncwarp();
#pragma unroll 4
    for (int r = 0; r < W2; ++r) {
      float t = 0.0f;
#pragma unroll
      for (int i = 0; i < W2; ++i) t = fmaf(ws.S[r * BS + i], ws.B[i * BS + col], t);
      jc[r] = fmaf(-0.5f, t, ws.S[r * BS + col]);
    }
  }
  __syncwarp();  // the ring aliases B and S
  // (3) A_ij <- A_ij J', V_ij <- V_ij J' (Alg 1 l.7)
  apply_f32<W2>(ws.ring, Wm, ld, mrows, I, J, lane, jc);
  apply_f32<W2>(ws.ring, Vm, ldv, vrows, I, J, lane, jc);
  return true;
}

// ---- Cross-CTA plumbing for a matrix spread over a thread-block cluster (tailoring) ----
// A matrix may be owned by a cluster of CL CTAs (CL = 1, 2, 4, 8; chosen by the planner from the batch
// composition, PAPER.md:228, 261-269 -- scheduling only, never arithmetic, Z22). The pairs of a
// round-robin step are spread over all CL x NW warps of the cluster; the per-block dataflow counters,
// the convergence vote and the finalisation arrays live in the shared memory of CTA rank 0 and are
// reached through distributed shared memory (generic addresses from map_shared_rank). W and V stay in
// the global (L2-resident) slot of the matrix; every pair's arithmetic is that of the one-CTA kernel,
// so results are bitwise independent of CL (tests/test_gpu_cluster.py).
__device__ __forceinline__ unsigned cl_rank() {
  unsigned r;
  asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
  return r;
}
__device__ __forceinline__ unsigned cl_nrank() {
  unsigned r;
  asm volatile("mov.u32 %0, %%cluster_nctarank;" : "=r"(r));
  return r;
}
__device__ __forceinline__ unsigned cl_id() {
  unsigned r;
  asm volatile("mov.u32 %0, %%clusterid.x;" : "=r"(r));
  return r;
}
// Cluster-wide barrier with release / acquire semantics (orders global and shared memory).
__device__ __forceinline__ void cl_sync() {
  asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}
// Generic address of `p` (a __shared__ variable) in the CTA of cluster rank 0.
template <typename T>
__device__ __forceinline__ T* at_rank0(T* p) {
  uint64_t g;
  asm volatile("mapa.u64 %0, %1, 0;" : "=l"(g) : "l"(reinterpret_cast<uint64_t>(p)));
  return reinterpret_cast<T*>(g);
}
// Dataflow counter of a column block: acquire-load / release-store at CTA scope (one CTA per matrix)
// or at cluster scope (the counter sits in rank 0's shared memory).
template <bool CLU>
__device__ __forceinline__ int ver_acquire(int* p) {
  if constexpr (CLU) {
    int v;  // an atomic read (atom.acquire, not ld.acquire): compute-sanitizer racecheck models atomics
    asm volatile("atom.acquire.cluster.or.b32 %0, [%1], 0;" : "=r"(v) : "l"(p) : "memory");
    return v;
  } else {
    return atomicAdd(p, 0);  // relaxed read; the fence after the spin orders the panel reads
  }
}
template <bool CLU>
__device__ __forceinline__ void ver_release(int* p, int v) {
  if constexpr (CLU) {
    int old;
    asm volatile("atom.release.cluster.exch.b32 %0, [%1], %2;" : "=r"(old) : "l"(p), "r"(v) : "memory");
  } else {
    atomicExch(p, v);
  }
}
template <bool CLU>
__device__ __forceinline__ void pair_fence() {
  if constexpr (CLU)
    __threadfence();  // the panels of the pair are read / written by warps on other SMs
  else
    __threadfence_block();
}

// Per-warp shared-memory stride: the pair buffers, or a 32 x 33 transpose tile for the stage-in.
template <int W2, typename TW = double>
__host__ __device__ constexpr size_t warp_stride() {
  constexpr size_t pb = sizeof(TW) == 8 ? WarpSmem<W2>::bytes() : WarpSmemF<W2>::bytes();
  return ((pb > 32 * 33 * sizeof(TW) ? pb : 32 * 33 * sizeof(TW)) + 15) & ~size_t(15);
}

}  // namespace

// MODE: kFlat (flat Gram path, one CTA per matrix), kFlatCluster (flat Gram path, a cluster of CTAs
// per matrix), kWcycle (Level 1 -> Level 2 recursion, one CTA). Separate instantiations keep one
// inlined copy of process_pair per kernel (register pressure).
enum { kFlat = 0, kFlatCluster = 1, kWcycle = 2, kPanel = 3 };

template <int W2, int NW, typename TI, typename TW, int MODE>
__global__ void __launch_bounds__(NW * 32, WCSVD_L1_MINB(NW)) l1_gram_kernel(const MatDesc* __restrict__ descs,
                                                             const int* __restrict__ order, SlotPool pool) {
  // TI: type of A, S, U, V in the caller's memory (double, or float for wcsvd_batched_f32); the
  // iteration always runs on the fp64 working copy. CLU: the matrix is owned by a CTA cluster.
  constexpr bool CLU = MODE == kFlatCluster;
  using C = PairCfg<W2>;
  const unsigned crank = CLU ? cl_rank() : 0u;
  const int CL = CLU ? (int)cl_nrank() : 1;
  const int mat = CLU ? (int)cl_id() : (int)blockIdx.x;
  const MatDesc d = descs[order[mat]];
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  constexpr int T = NW * 32;
  const int gw = (int)crank * NW + warp;  // warp id inside the matrix's cluster
  const int NWT = CL * NW;                // warps working on the matrix
  const int M = d.M, N = d.N, mp = d.m_pad, np = d.n_pad;

  extern __shared__ __align__(16) unsigned char smem_raw[];
  // TW: the working precision: fp64 (DMMA contractions; also the default for fp32 data, see launch_l1)
  // or fp32 (the FFMA path of wcsvd_batched_f32 with opts->f32_compute = 1)
  constexpr bool F32 = sizeof(TW) == 4;
  WarpSmem<W2> ws;
  WarpSmemF<W2> wsf;
  {
    unsigned char* p = smem_raw + warp * warp_stride<W2, TW>();
    if constexpr (F32) {
      wsf.B = reinterpret_cast<float*>(p);
      wsf.S = wsf.B + W2 * WarpSmemF<W2>::BS;
      wsf.ring = wsf.B;
      wsf.cs = reinterpret_cast<float2*>(p + WarpSmemF<W2>::region());
    } else {
      ws.B = reinterpret_cast<double*>(p);
      ws.S = ws.B + W2 * C::BS;
      ws.ring = ws.B;
      ws.cs = reinterpret_cast<double2*>(p + WarpSmem<W2>::region());
      ws.tt = reinterpret_cast<double*>(ws.cs + W2 / 2);
      ws.pq = reinterpret_cast<int2*>(ws.tt + W2 / 2);
    }
  }
  // Matrix-wide state (rank 0's copy is the one in use when CLU).
  __shared__ int s_flags[4];          // [0, 1] sweep votes (parity), [2] non-finite, [3] needs completion
  __shared__ int s_inner;             // total inner sweeps
  __shared__ int s_slot;              // workspace slot of the matrix
  __shared__ int s_grp[2 * NW];       // W-cycle group votes
  __shared__ int s_blkver[1024 / 8];  // per-block completed-pair counters (flat path)
  __shared__ unsigned long long s_max;
  __shared__ unsigned long long s_clmax[8];  // rank 0: per-CTA max |a_ij| (bit 63 = non-finite seen)
  __shared__ EvdMap<W2> s_em[32];     // inner-EVD work map per lane (per CTA)
  if (tid < 32) s_em[tid].init(tid);
  if (tid < 4) s_flags[tid] = 0;
  if (tid < 2 * NW) s_grp[tid] = 0;
  const int nb = np / C::W;
  for (int b = tid; b < nb; b += T) s_blkver[b] = 0;
  if (tid == 0) {
    s_inner = 0;
    s_max = 0ull;
    if (crank == 0) s_slot = slot_acquire(pool);
  }
  int* flags0 = s_flags;
  int* ver0 = s_blkver;
  int* inner0 = &s_inner;
  if constexpr (CLU) {
    flags0 = at_rank0(s_flags);
    ver0 = at_rank0(s_blkver);
    inner0 = at_rank0(&s_inner);
    cl_sync();
  } else {
    __syncthreads();
  }
  const int slot = CLU ? *at_rank0(&s_slot) : s_slot;
  TW* Wm = reinterpret_cast<TW*>(pool.base + (size_t)slot * pool.slot_doubles);
  TW* Vm = Wm + (size_t)mp * np;

  // ---- Stage-in: W = A or A^T, zero-padded to m_pad x n_pad; V = I. 32 x 32 tiles
  // per warp; the transpose (m < n) goes through a shared-memory tile so that both the reads of A
  // and the writes of W are coalesced. ----
  bool bad = false;
  double amax = 0.0;
#ifdef WCSVD_EXP_STAGE_OLD
  if (!CLU) {
    for (size_t e = tid; e < (size_t)mp * np; e += T) {
      const int c = (int)(e / mp), r = (int)(e % mp);
      double v = 0.0;
      if (r < M && c < N) {
        const TI* Ain = reinterpret_cast<const TI*>(d.A);
        v = (double)(d.swapped ? Ain[(size_t)r * d.lda + c] : Ain[(size_t)c * d.lda + r]);
        bad |= !isfinite(v);
        amax = fmax(amax, fabs(v));
      }
      Wm[e] = v;
    }
  } else
#endif
  {
    const TI* Ain = reinterpret_cast<const TI*>(d.A);
    TW* tile = reinterpret_cast<TW*>(smem_raw + warp * warp_stride<W2, TW>());
    const int ntr = (mp + 31) / 32, ntc = (np + 31) / 32;
    for (int t = gw; t < ntr * ntc; t += NWT) {
      const int r0 = (t % ntr) * 32, c0 = (t / ntr) * 32;
      if (d.swapped) {
        // W row r = A column r; lane -> A row c0 + lane (contiguous)
        for (int rr = 0; rr < 32; ++rr) {
          const int r = r0 + rr, c = c0 + lane;
          double v = 0.0;
          if (r < M && c < N) {
            v = (double)Ain[(size_t)r * d.lda + c];
            bad |= !isfinite(v);
            amax = fmax(amax, fabs(v));
          }
          tile[rr * 33 + lane] = (TW)v;
        }
        __syncwarp();
        for (int cc = 0; cc < 32; ++cc) {
          const int c = c0 + cc, r = r0 + lane;
          if (r < mp && c < np) Wm[(size_t)c * mp + r] = tile[lane * 33 + cc];
        }
        __syncwarp();
      } else {
        for (int cc = 0; cc < 32; ++cc) {
          const int c = c0 + cc, r = r0 + lane;
          if (r < mp && c < np) {
            double v = 0.0;
            if (r < M && c < N) {
              v = (double)Ain[(size_t)c * d.lda + r];
              bad |= !isfinite(v);
              amax = fmax(amax, fabs(v));
            }
            Wm[(size_t)c * mp + r] = (TW)v;
          }
        }
      }
    }
  }
  if (d.withv)
    for (size_t e = (size_t)crank * T + tid; e < (size_t)np * np; e += (size_t)CL * T)
      Vm[e] = ((int)(e % np) == (int)(e / np)) ? TW(1) : TW(0);
  const int vrows = d.withv ? np : 0;  // values / U-only mode: V_x is not accumulated (§8(f4))
  // max |a_ij| and the non-finite flag: CTA-local atomics, then (cluster) one slot per CTA in rank 0
  if (bad) atomicOr(&s_flags[2], 1);
  if (amax > 0.0) atomicMax(&s_max, (unsigned long long)__double_as_longlong(amax));
  __syncthreads();
  bool nonfinite = s_flags[2] != 0;
  unsigned long long gmax = s_max;
  if constexpr (CLU) {
    if (tid == 0) at_rank0(s_clmax)[crank] = gmax | (nonfinite ? (1ull << 63) : 0ull);
    cl_sync();
    const unsigned long long* cm = at_rank0(s_clmax);
    gmax = 0ull;
    for (int r = 0; r < CL; ++r) gmax = (cm[r] & ~(1ull << 63)) > gmax ? (cm[r] & ~(1ull << 63)) : gmax;
    nonfinite = false;
    for (int r = 0; r < CL; ++r) nonfinite |= (cm[r] >> 63) != 0;
  }
  // Exact power-of-two pre-scaling to max|w| in [0.5, 1) (see l0_jacobi.cu); every
  // warp scales the tiles it wrote.
  int sexp = 0;
  if (!nonfinite && gmax != 0ull) {
    frexp(__longlong_as_double((long long)gmax), &sexp);
    const double f = ldexp(1.0, -sexp);
    const int ntr = (mp + 31) / 32, ntc = (np + 31) / 32;
    for (int t = gw; t < ntr * ntc; t += NWT) {
      const int r0 = (t % ntr) * 32, c0 = (t / ntr) * 32, r = r0 + lane;
      if (r < mp)
        for (int cc = 0; cc < 32 && c0 + cc < np; ++cc) Wm[(size_t)(c0 + cc) * mp + r] *= (TW)f;
    }
  }
  if constexpr (CLU) cl_sync(); else __syncthreads();
  const TW tol2 = (TW)(d.tol * d.tol);

  int sweep = 0;
  bool converged = false;
  int my_inner = 0;
  if (MODE != kWcycle && !nonfinite) {
    // Flat Level 1: round-robin over the n_pad / w column blocks (Alg 1). Pairs are
    // scheduled by dataflow instead of a barrier per step: ver[b] counts the pairs block b has
    // completed, and the pair (I, J) of global step g starts once both blocks reached g. Each warp
    // takes its pairs in (step, pair) order, so waits only point backwards (no deadlock), and warps
    // drift into different phases (EVD overlaps other warps' DMMA work). The arithmetic of every pair
    // is unchanged, so the result is bitwise that of a barrier schedule on any number of CTAs.
    int gstep = 0;
    while (sweep < d.max_sweeps) {
      bool rot_any = false;
      for (int step = 0; step < nb - 1; ++step, ++gstep) {
        for (int p = gw; p < nb / 2; p += NWT) {
          const int I = rr_content(2 * p, step, nb), J = rr_content(2 * p + 1, step, nb);
          if (lane == 0) {  // acquire
            while (ver_acquire<CLU>(&ver0[I]) < gstep || ver_acquire<CLU>(&ver0[J]) < gstep) __nanosleep(20);
          }
          __syncwarp();
          pair_fence<CLU>();  // the previous owners' W / V writes are visible to every lane
          if constexpr (F32)
            rot_any |= process_pair_f32<W2>(wsf, Wm, mp, mp, Vm, np, vrows, I, J, tol2, d.inner_cap, lane, &my_inner);
          else
            rot_any |= process_pair<W2, MODE == kPanel>(ws, s_em, Wm, mp, mp, Vm, np, vrows, I, J, tol2, d.inner_cap,
                                                        lane, &my_inner);
          pair_fence<CLU>();  // every lane's W / V writes precede ...
          __syncwarp();
          if (lane == 0) {    // ... the release
            ver_release<CLU>(&ver0[I], gstep + 1);
            ver_release<CLU>(&ver0[J], gstep + 1);
          }
        }
      }
      ++sweep;
      if (rot_any && lane == 0) atomicOr(&flags0[sweep & 1], 1);
      if constexpr (CLU) cl_sync(); else __syncthreads();
      const bool any = (CLU ? *(volatile int*)&flags0[sweep & 1] : s_flags[sweep & 1]) != 0;
      if constexpr (CLU) cl_sync(); else __syncthreads();
      if (crank == 0 && tid == 0) s_flags[sweep & 1] = 0;
      if (!any) { converged = true; break; }
    }
#ifdef WCSVD_EXP_FLAT_WITH_WCYCLE
  } else if ((MODE == kWcycle || (MODE == kFlat && d.w2 != 0)) && !nonfinite) {
#else
  } else if (MODE == kWcycle && !nonfinite) {
#endif
    // W-cycle (Alg 2 l.12-14; Step 3; Fig 3-4): Level-1 super-blocks
    // of width w1 = d.w are paired round-robin; each super-pair panel [A_I A_J] (M x 2 w1) fits no
    // on-chip EVD, so it recurses to Level 2: block Jacobi with w2 = d.w2 (the EVD width W2/2) over
    // its 2r sub-blocks (r = w1 / w2) until they are mutually orthogonal or inner_cap2 Level-2
    // sweeps ran. The Level-2 rotations are applied to the A and V sub-panels as they are found, so
    // the panel leaves Level 2 already rotated and V carries J_IJ (Z23: no separate A update).
    // A group of GS warps owns one super-pair; named barriers separate its Level-2 steps.
    const int r = d.w / C::W;
    const int nb1 = np / d.w;
    const int GS = (r < NW) ? r : NW, NG = NW / GS;
    const int grp = warp / GS, gwi = warp % GS;
    const bool active_grp = grp < NG;
    while (sweep < d.max_sweeps) {
      bool rot_any = false;
      for (int s1 = 0; s1 < nb1 - 1; ++s1) {
        if (active_grp) {
          for (int p1 = grp; p1 < nb1 / 2; p1 += NG) {
            const int I1 = rr_content(2 * p1, s1, nb1), J1 = rr_content(2 * p1 + 1, s1, nb1);
            for (int isw = 0; isw < d.inner_cap2; ++isw) {
              bool mine = false;
              for (int s2 = 0; s2 < 2 * r - 1; ++s2) {
                for (int p2 = gwi; p2 < r; p2 += GS) {
                  const int a = rr_content(2 * p2, s2, 2 * r), b = rr_content(2 * p2 + 1, s2, 2 * r);
                  const int Ia = (a < r) ? I1 * r + a : J1 * r + (a - r);
                  const int Ib = (b < r) ? I1 * r + b : J1 * r + (b - r);
                  if constexpr (F32)
                    mine |= process_pair_f32<W2>(wsf, Wm, mp, mp, Vm, np, vrows, Ia, Ib, tol2, d.inner_cap, lane, &my_inner);
                  else
                    mine |= process_pair<W2>(ws, s_em, Wm, mp, mp, Vm, np, vrows, Ia, Ib, tol2, d.inner_cap, lane, &my_inner);
                }
                named_bar(1 + grp, GS * 32);
              }
              // group vote on "some Level-2 pair rotated in this inner sweep"
              if (mine && lane == 0) s_grp[grp * 2 + (isw & 1)] = 1;
              named_bar(1 + grp, GS * 32);
              const bool any2 = s_grp[grp * 2 + (isw & 1)] != 0;
              named_bar(1 + grp, GS * 32);
              if (gwi == 0 && lane == 0) s_grp[grp * 2 + (isw & 1)] = 0;
              rot_any |= any2;
              if (!any2) break;
            }
          }
        }
        __syncthreads();
      }
      ++sweep;
      if (rot_any && lane == 0) s_flags[sweep & 1] = 1;
      __syncthreads();
      const bool any = s_flags[sweep & 1] != 0;
      __syncthreads();
      if (tid == 0) s_flags[sweep & 1] = 0;
      if (!any) { converged = true; break; }
    }
  }
  if (lane == 0 && my_inner) atomicAdd(inner0, my_inner);

  // ---- Finalisation: sigma, rank, sign (Z15), U = W / sigma, un-orientation. ----
  // sigma and the sign of every column go to rank 0's arrays; every CTA then copies them locally.
  // one CTA: reuse the warp buffers; cluster: a dedicated region after them (other CTAs write rank 0's
  // copy while its warps may still be draining their slab rings)
  double* s_sig = reinterpret_cast<double*>(smem_raw + (CLU ? NW * warp_stride<W2, TW>() : 0));  // [N]
  double* s_sgn = s_sig + N;                             // [N]
  double* sig0 = s_sig;
  double* sgn0 = s_sgn;
  if constexpr (CLU) {
    sig0 = at_rank0(s_sig);
    sgn0 = at_rank0(s_sgn);
  } else {
    __syncthreads();
  }
  for (int j = gw; j < N; j += NWT) {
    const TW* col = Wm + (size_t)j * mp;
    double a = 0.0;
    for (int r = lane; r < M; r += 32) {
      const double x = (double)__ldcg(col + r);
      a = fma(x, x, a);
    }
    for (int off = 16; off > 0; off >>= 1) a += __shfl_xor_sync(0xffffffffu, a, off);
    // Z15 sign rule on the square factor V_x; without V (values / U-only mode) on the columns of X.
    const TW* vc = d.withv ? Vm + (size_t)j * np : col;
    const int vlen = d.withv ? N : M;
    double best = 0.0;
    int bi = 0x7fffffff;
    for (int i = lane; i < vlen; i += 32) {
      const double v = (double)__ldcg(vc + i);
      if (fabs(v) > fabs(best)) { best = v; bi = i; }
    }
    for (int off = 16; off > 0; off >>= 1) {
      const double ob = __shfl_xor_sync(0xffffffffu, best, off);
      const int oi = __shfl_xor_sync(0xffffffffu, bi, off);
      if (fabs(ob) > fabs(best) || (fabs(ob) == fabs(best) && oi < bi)) { best = ob; bi = oi; }
    }
    if (lane == 0) {
      sig0[j] = nonfinite ? __longlong_as_double(0x7ff8000000000000ULL) : sqrt(a);
      sgn0[j] = (best < 0.0) ? -1.0 : 1.0;
    }
  }
  if constexpr (CLU) {
    cl_sync();
    if (crank != 0)
      for (int j = tid; j < N; j += T) {
        s_sig[j] = sig0[j];
        s_sgn[j] = sgn0[j];
      }
  }
  __syncthreads();
  double sig1 = 0.0;
  for (int i = 0; i < N; ++i) sig1 = fmax(sig1, s_sig[i]);
  const double thresh = sig1 * (double)M * (F32 ? 5.9604644775390625e-08 : kU53);  // Z14: the working precision's u
  const double nanv = __longlong_as_double(0x7ff8000000000000ULL);
  TI* dstW = reinterpret_cast<TI*>(d.swapped ? d.V : d.U);
  const int ldW = d.swapped ? d.ldv : d.ldu;
  TI* dstV = reinterpret_cast<TI*>(d.swapped ? d.U : d.V);
  const int ldV = d.swapped ? d.ldu : d.ldv;
  bool needs_completion = false;
  for (int j = gw; j < N; j += NWT) {
    // rank of column j in the stable descending order (ties to the lower index)
    const double sj = s_sig[j], sgn = s_sgn[j];
    int rk = 0;
    if (nonfinite) {
      rk = j;
    } else {
      for (int i = lane; i < N; i += 32) {
        const double si = s_sig[i];
        rk += (si > sj) || (si == sj && i < j);
      }
      for (int off = 16; off > 0; off >>= 1) rk += __shfl_xor_sync(0xffffffffu, rk, off);
    }
    const bool ok = sj > thresh;
    needs_completion |= !ok;
    if (dstW) {
      const TW* col = Wm + (size_t)j * mp;
      for (int r = lane; r < M; r += 32)
        dstW[(size_t)rk * ldW + r] = (TI)(nonfinite ? nanv : (ok ? sgn * ((double)__ldcg(col + r) / sj) : sgn * 0.0));
    }
    if (dstV) {
      const TW* vc = Vm + (size_t)j * np;
      for (int i = lane; i < N; i += 32) dstV[(size_t)rk * ldV + i] = (TI)(nonfinite ? nanv : sgn * (double)__ldcg(vc + i));
    }
    if (lane == 0) reinterpret_cast<TI*>(d.S)[rk] = (TI)(nonfinite ? sj : ldexp(sj, sexp));
  }
  if (needs_completion && !nonfinite && lane == 0) atomicOr(&flags0[3], 1);
  if constexpr (CLU) cl_sync(); else __syncthreads();
  if (crank == 0 && tid == 0) {
    if (d.info) d.info[d.idx] = nonfinite ? -2 : (converged ? sweep : -1);
    if (d.sweeps_inner) d.sweeps_inner[d.idx] = s_inner;
    if (d.status) d.status[d.idx] = (s_flags[3] && dstW) ? kNeedsCompletion : 0;
    slot_release(pool, s_slot);
  }
}

template <int W2, int NW, typename TI, typename TW, int MODE>
static cudaError_t launch_l1_t(const MatDesc* descs, const int* order, int count, int cluster, const SlotPool& pool,
                               cudaStream_t stream) {
  size_t smem = NW * warp_stride<W2, TW>();
  const size_t fin = 2 * 8 * 1024;  // finalisation arrays: alias the warp buffers (one CTA) or follow them
  if (MODE == kFlatCluster) smem += fin;
  else if (smem < fin) smem = fin;
  auto kern = l1_gram_kernel<W2, NW, TI, TW, MODE>;
  cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  if (MODE != kFlatCluster) {
    kern<<<count, NW * 32, smem, stream>>>(descs, order, pool);
    return cudaGetLastError();
  }
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((unsigned)(count * cluster), 1, 1);
  cfg.blockDim = dim3(NW * 32, 1, 1);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = stream;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeClusterDimension;
  at[0].val.clusterDim.x = (unsigned)cluster;
  at[0].val.clusterDim.y = 1;
  at[0].val.clusterDim.z = 1;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  return cudaLaunchKernelEx(&cfg, kern, descs, order, pool);
}

template <typename TI, typename TW, int W2, int NW>
static cudaError_t launch_l1_m(int wcycle, const MatDesc* descs, const int* order, int count, int cluster,
                               const SlotPool& pool, cudaStream_t stream) {
  if (wcycle == 2) {  // group (i) PANEL path: fp64, 2w = 32
    if constexpr (W2 == 32 && sizeof(TW) == 8) return launch_l1_t<W2, NW, TI, TW, kPanel>(descs, order, count, 1, pool, stream);
    return cudaErrorInvalidValue;
  }
  if (wcycle) return launch_l1_t<W2, NW, TI, TW, kWcycle>(descs, order, count, 1, pool, stream);
  if (cluster > 1) return launch_l1_t<W2, NW, TI, TW, kFlatCluster>(descs, order, count, cluster, pool, stream);
  return launch_l1_t<W2, NW, TI, TW, kFlat>(descs, order, count, 1, pool, stream);
}

template <typename TI, typename TW>
static cudaError_t launch_l1_v(int variant, int wcycle, const MatDesc* descs, const int* order, int count,
                               int cluster, const SlotPool& pool, cudaStream_t stream) {
  switch (variant) {
    case kL1_16x4: return launch_l1_m<TI, TW, 16, 4>(wcycle, descs, order, count, cluster, pool, stream);
    case kL1_32x4: return launch_l1_m<TI, TW, 32, 4>(wcycle, descs, order, count, cluster, pool, stream);
    case kL1_32x8: return launch_l1_m<TI, TW, 32, 8>(wcycle, descs, order, count, cluster, pool, stream);
    default: return cudaErrorInvalidValue;
  }
}

// fp32 data: f32_compute = 0 iterates on an fp64 working copy with the DMMA contractions (B200: 239 /
// 361 ms on C3 / C4 as fp32), 1 on an fp32 working copy with FFMA contractions (447 / 1011 ms: FFMA
// needs 8x the issue slots of DMMA per flop and the FP32 pipe is only 2x the FP64 one -- profiles/
// f32_paths_r02.json), so the planner default is 0.
cudaError_t launch_l1(int variant, int wcycle, int fp32, int f32_compute, const MatDesc* descs, const int* order,
                      int count, int cluster, const SlotPool& pool, cudaStream_t stream) {
  if (!fp32) return launch_l1_v<double, double>(variant, wcycle, descs, order, count, cluster, pool, stream);
  return f32_compute ? launch_l1_v<float, float>(variant, wcycle, descs, order, count, cluster, pool, stream)
                     : launch_l1_v<float, double>(variant, wcycle, descs, order, count, cluster, pool, stream);
}

}  // namespace wcsvd

#ifdef WCSVD_PHASE_PROFILE
// Debug builds only: copy (and optionally reset) the per-phase cycle totals of the Level-1 kernel.
extern "C" WCSVD_API int wcsvd_debug_phase_cycles(unsigned long long* out, int reset) {
  if (cudaMemcpyFromSymbol(out, wcsvd::g_phase_cycles, sizeof(unsigned long long) * 12) != cudaSuccess) return -1;
  if (reset) {
    unsigned long long z[12] = {0, 0, 0, 0, 0, 0, 0, 0, 0, 0, 0, 0};
    cudaMemcpyToSymbol(wcsvd::g_phase_cycles, z, sizeof(z));
  }
  return 0;
}
#endif
