/* oracle.c -- CPU ORACLE. TEST INFRASTRUCTURE ONLY.
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference legs may
 * load this library. The product path (paper_conf_sc_xiaopxsmmlzt22_b200/, libwcsvd.so) never
 * links, imports or calls it, and it shares no code, header, table or constant with the CUDA path.
 *
 * What it computes (the plain definition): the economy SVD A = U diag(S) V^T of
 * each input, by a textbook cyclic one-sided Jacobi iteration in long double (x87, 64-bit
 * mantissa) -- PAPER.md:47-58 (§II.A eq 1-2), PAPER.md:72-84 (§II.C eq 3-4)
 * (§IV.B transpose), PAPER.md:181 (§III.C finalisation). See oracle_body.inc for the steps.
 *
 * Also: a textbook cyclic two-sided Jacobi EVD of a symmetric matrix (§II.D eq 5),
 * the sequential reference for the parallel round-robin EVD (§IV.C).
 *
 * Pins (tests/test_oracle.py, -m "not gpu"): 2x2 closed form (P1), diagonal / permuted diagonal
 * (P7), prescribed spectra Q1 diag(s) Q2^T (P8), sum sigma^2 = ||A||_F^2 and orthogonality (P9),
 * power-of-two scaling bitwise (P10), transpose symmetry (P11), brute-force eigenvalues of A^T A
 * and LAPACK svd cross-check (P6), rank-deficient completion (Z14). Build: gcc -O2 -fopenmp -shared.
 */
#include <math.h>
#include <omp.h>
#include <stdlib.h>
#include <string.h>

/* ---- long double instantiation: the parity oracle ---- */
#define REAL long double
#define SUFFIX ld
#define SQRT sqrtl
#define FABS fabsl
#define EPS_REAL 5.42101086242752217004e-20L /* 2^-64: unit roundoff of the x87 64-bit mantissa */
#include "oracle_body.inc"
#undef REAL
#undef SUFFIX
#undef SQRT
#undef FABS
#undef EPS_REAL

/* ---- double instantiation: the same code, timed as the CPU baseline ---- */
#define REAL double
#define SUFFIX d
#define SQRT sqrt
#define FABS fabs
#define EPS_REAL 1.1102230246251565404e-16 /* 2^-53 */
#include "oracle_body.inc"
#undef REAL
#undef SUFFIX
#undef SQRT
#undef FABS
#undef EPS_REAL

/* Two-sided cyclic Jacobi EVD of a symmetric n x n B (column-major, ld n), long double.
 * PAPER.md:93-99 (§II.D): for a pair (i,j), rho = (b_ii - b_jj)/(2 b_ij),
 * t = sign(rho)/(|rho| + sqrt(1+rho^2)), c = 1/sqrt(1+t^2), s = t c, G = [[c,-s],[s,c]] on
 * rows/cols (i,j): B <- G^T B G, J <- J G (PAPER.md:93 J = G_1 G_2 ...). Threshold Jacobi (Z8):
 * a pair rotates only if |b_ij| > tol * sqrt(|b_ii|) * sqrt(|b_jj|). Converged when a sweep has no
 * rotation. Outputs: lambda[n] = diag of the final B (unsorted), J (n x n, ld n). Returns sweeps
 * (> 0) or -1 when max_sweeps was hit. */
int oracle_syevj_ld(int n, const double* B_in, double tol_in, int max_sweeps, double* lambda,
                    double* J_out) {
  long double* B = (long double*)malloc(sizeof(long double) * (size_t)n * (size_t)n);
  long double* J = (long double*)malloc(sizeof(long double) * (size_t)n * (size_t)n);
  if (!B || !J) { free(B); free(J); return -2; }
  for (size_t e = 0; e < (size_t)n * n; ++e) B[e] = (long double)B_in[e];
  for (int c = 0; c < n; ++c)
    for (int r = 0; r < n; ++r) J[(size_t)c * n + r] = (r == c) ? 1 : 0;
  const long double tol = (tol_in > 0) ? (long double)tol_in : sqrtl((long double)n) * 5.42101086242752217004e-20L;
  if (max_sweeps <= 0) max_sweeps = 60;
  int sweeps = 0, converged = 0;
  while (sweeps < max_sweeps) {
    ++sweeps;
    long long rot = 0;
    for (int i = 0; i < n - 1; ++i) {
      for (int j = i + 1; j < n; ++j) {
        const long double bii = B[(size_t)i * n + i], bjj = B[(size_t)j * n + j];
        const long double bij = B[(size_t)j * n + i];
        if (bij == 0) continue;
        if (fabsl(bij) <= tol * sqrtl(fabsl(bii)) * sqrtl(fabsl(bjj))) continue;
        const long double rho = (bii - bjj) / (2 * bij);
        const long double sg = (rho >= 0) ? 1.0L : -1.0L;
        const long double t = sg / (fabsl(rho) + sqrtl(1 + rho * rho));
        const long double c = 1 / sqrtl(1 + t * t);
        const long double s = t * c;
        /* B <- B G (columns i, j) */
        for (int r = 0; r < n; ++r) {
          const long double x = B[(size_t)i * n + r], y = B[(size_t)j * n + r];
          B[(size_t)i * n + r] = c * x + s * y;
          B[(size_t)j * n + r] = -s * x + c * y;
        }
        /* B <- G^T B (rows i, j) */
        for (int cc = 0; cc < n; ++cc) {
          const long double x = B[(size_t)cc * n + i], y = B[(size_t)cc * n + j];
          B[(size_t)cc * n + i] = c * x + s * y;
          B[(size_t)cc * n + j] = -s * x + c * y;
        }
        /* J <- J G */
        for (int r = 0; r < n; ++r) {
          const long double x = J[(size_t)i * n + r], y = J[(size_t)j * n + r];
          J[(size_t)i * n + r] = c * x + s * y;
          J[(size_t)j * n + r] = -s * x + c * y;
        }
        ++rot;
      }
    }
    if (rot == 0) { converged = 1; break; }
  }
  for (int i = 0; i < n; ++i) lambda[i] = (double)B[(size_t)i * n + i];
  if (J_out)
    for (size_t e = 0; e < (size_t)n * n; ++e) J_out[e] = (double)J[e];
  free(B); free(J);
  return converged ? sweeps : -1;
}

/* OpenMP thread count of the batched drivers (set explicitly: launchers such as torchrun export
 * OMP_NUM_THREADS=1), and the count actually in effect. */
void oracle_set_threads(int n) { if (n > 0) omp_set_num_threads(n); }
int oracle_get_threads(void) { return omp_get_max_threads(); }

/* Mantissa bits of long double on this host (tests assert 64 for the x87 format). */
int oracle_ldbl_mant_dig(void) { return __LDBL_MANT_DIG__; }
