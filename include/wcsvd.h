/* wcsvd.h -- C-ABI of the B200-native batched one-sided Jacobi SVD (W-cycle SVD hot path).
 *
 * Library: paper_conf_sc_xiaopxsmmlzt22_b200/libwcsvd.so, CUDA for sm_100a only.
 * Citations are lines of the paper's text, PAPER.md:N (section / equation / algorithm).
 *
 * Problem (§II.A eq 1; §III.B; Alg 2 l.1):
 *   a batch of mu independent real matrices A^k (m_k x n_k, sizes may all differ) is factorised
 *   as A^k = U^k diag(S^k) (V^k)^T -- economy form, k_k = min(m_k, n_k) triplets.
 * Method (the hot path, BASELINE.json north_star): batched one-sided Jacobi. Column-block pairs
 *   [A_i A_j] are orthogonalised by Gram -> in-SMEM Jacobi EVD -> A/V block update -> off-norm test
 *   (Alg 1; Alg 2), inside the multilevel W-cycle;
 *   matrices that fit on-chip run the Level-0 vector-rotation kernel (§IV.B).
 *
 * Conventions (all entry points):
 *  - fp64, column-major, economy SVD: S[k] descending, U m x k, V n x k.
 *  - Ownership: the caller owns A, S, U, V (DEVICE memory) and every host array; host arrays are
 *    consumed before the call returns and may be freed immediately. The library owns only its
 *    workspace: stream-ordered allocations on `stream` from a memory pool the library creates for
 *    the device (never the device's default pool; freed blocks stay cached in that pool until
 *    wcsvd_trim_workspace), or the caller's buffer via _ex. The working copies W, V of Level >= 1
 *    matrices (and the Level-0 park buffers) come from slot pools sized to the CTAs that can be
 *    resident at once, not to the batch. A is read-only.
 *  - Asynchronous on `stream`: a return of WCSVD_OK means the work was enqueued.
 *  - Errors: negative codes are returned synchronously and nothing is enqueued on failure:
 *      -i          the i-th argument (1-based) is invalid (LAPACK convention);
 *      WCSVD_ENOTSUP  a size outside 1 <= m, n <= 1024;
 *      WCSVD_ECUDA    a CUDA error (no device, launch failure, missing sm_100a image);
 *      WCSVD_ENOMEM   workspace allocation failed.
 *    Numerical outcomes are per matrix, asynchronous, in opts->info (see wcsvd_opts).
 *  - Deterministic: the outputs for one matrix depend only on (m, n, the bits of A, tol,
 *    max_sweeps) -- never on batch composition, stream, device index or device count. The plan is
 *    a function of (m, n) only; there are no floating-point atomics.
 *  - Reentrant. Process-wide state: only the per-device workspace pool above (created once, guarded
 *    by a mutex), the planner's immutable table coordinates, and, per host thread and device, the
 *    streams / events of wcsvd_batched_host's pipeline (created on first use, drained by every call,
 *    never shared between threads); nothing a call does changes another call's results.
 */
#ifndef WCSVD_H_
#define WCSVD_H_

#include <stddef.h>

#if defined(__GNUC__)
#define WCSVD_API __attribute__((visibility("default")))
#else
#define WCSVD_API
#endif

#ifdef __cplusplus
extern "C" {
#endif

/* cudaStream_t is an opaque pointer; declared here so this header needs no CUDA include. */
typedef struct CUstream_st* wcsvd_stream_t;

enum {
  WCSVD_OK = 0,
  WCSVD_ENOTSUP = -100,
  WCSVD_ECUDA = -101,
  WCSVD_ENOMEM = -102
};

/* Paths a matrix can take through the W-cycle (Alg 2 l.2-14). */
enum {
  WCSVD_PATH_AUTO = 0,
  WCSVD_PATH_L0 = 1,      /* whole matrix on-chip: vector-rotation Jacobi, Alg 2 l.2-3 */
  WCSVD_PATH_GRAM = 2,    /* Level 1: Gram -> EVD(B_ij) -> GEMM update, Alg 2 l.10-11 */
  WCSVD_PATH_WCYCLE = 3,  /* Level 1 -> Level 2 recursion on each pair panel, Alg 2 l.12-14 */
  WCSVD_PATH_PANEL = 4    /* Level 1, J from the SVD of the pair panel (group (i), Alg 2 l.8-9): one-sided
                             Jacobi of its CholeskyQR factor R (2w x 2w) in registers; w = 16, fp64 */
};

/* wcsvd_batched -- batched economy SVD.
 *  batch       >= 0; 0 is a no-op returning WCSVD_OK.                                    (arg 1)
 *  m, n        host arrays [batch]; 1 <= m[b], n[b] <= 1024 (else WCSVD_ENOTSUP).        (2, 3)
 *  A           host array [batch] of DEVICE pointers; A[b] is m x n column-major, ld lda[b],
 *              8-byte aligned; not modified. Must not alias S/U/V.                        (4)
 *  lda         host array [batch]; lda[b] >= m[b].                                        (5)
 *  S           host array [batch] of DEVICE pointers to k = min(m,n) doubles, descending.   (6)
 *  U           NULL (left vectors not returned) or host array [batch] of DEVICE pointers
 *              (entries may be NULL): m x k column-major, ld m.                           (7)
 *  V           NULL or host array [batch] of DEVICE pointers: n x k column-major, ld n.  (8)
 *  tol         relative orthogonality threshold |a_i^T a_j| <= tol ||a_i|| ||a_j||;
 *              <= 0 -> sqrt(max(m,n)) * 2^-53 per matrix.                                (9)
 *  max_sweeps  outer-sweep cap; <= 0 -> 60. When reached, the best iterate is finalised (Z26). (10)
 *  stream      CUDA stream (cudaStream_t) the work is enqueued on; NULL = legacy default. (11)
 * Returns WCSVD_OK or a negative code (above). */
WCSVD_API int wcsvd_batched(int batch, const int* m, const int* n, const double* const* A, const int* lda,
                  double* const* S, double* const* U, double* const* V, double tol, int max_sweeps,
                  wcsvd_stream_t stream);

/* Extended options (argument 12 of wcsvd_batched_ex). Zero-initialise, then set struct_size. */
typedef struct {
  size_t struct_size;      /* = sizeof(wcsvd_opts); ABI versioning */
  const int* ldu;          /* host [batch] or NULL (-> m): leading dimensions of U[b], >= m[b] */
  const int* ldv;          /* host [batch] or NULL (-> n): leading dimensions of V[b], >= n[b] */
  int* info;               /* DEVICE int[batch] or NULL. Per matrix, written asynchronously:
                              > 0  outer sweeps used (the last, rotation-free one included, Z24);
                              -1   not converged within max_sweeps (best iterate returned, Z26);
                              -2   non-finite input (S, U, V filled with NaN). */
  int* sweeps_inner;       /* DEVICE int[batch] or NULL: total inner (Level >= 2 / EVD) sweeps */
  void* workspace;         /* DEVICE buffer or NULL (-> stream-ordered internal allocation) */
  size_t workspace_bytes;  /* size of `workspace`; must be >= wcsvd_workspace_size(...) */
  int force_path;          /* 0 = planner; else WCSVD_PATH_* for every matrix (ablations) */
  int force_w;             /* 0 = planner; else the EVD block width w in {8, 16} (Level 1 of the
                              Gram path, Level 2 of the W-cycle path) */
  int wcycle_sweeps;       /* 0 = planner (2); cap on Level-2 sweeps per W-cycle super-pair */
  int inner_sweeps;        /* 0 = planner (1); cap on EVD sweeps per pair */
  int pair_warps;          /* 0 or 1: warps per column-block pair (the two-warp ablation executor of
                              round 1 was removed; any other value is -12) */
  int cluster_ctas;        /* 0 = planner (tailoring: a Gram-path matrix whose one-CTA time would
                              dominate the batch is spread over a thread-block cluster of 2, 4 or 8
                              CTAs); 1, 2, 4, 8 force the CTAs per Gram-path matrix (ablations).
                              Results are bitwise independent of it. Other values: -12 */
  int f32_compute;         /* wcsvd_batched_f32 only: 0 = planner (Gram-path matrices iterate on an fp64
                              working copy with FP64 DMMA contractions and are rounded at finalisation:
                              the fastest on B200), 1 = iterate in fp32 (FFMA Gram / update, fp32 EVD and
                              Newton-Schulz on an fp32 working copy; ablation). Other values: -12 */
} wcsvd_opts;

WCSVD_API int wcsvd_batched_ex(int batch, const int* m, const int* n, const double* const* A, const int* lda,
                     double* const* S, double* const* U, double* const* V, double tol,
                     int max_sweeps, wcsvd_stream_t stream, const wcsvd_opts* opts);

/* wcsvd_batched_f32 / _f32_ex -- the fp32 variant: same arguments, layout,
 * ownership, errors and determinism as wcsvd_batched, with float data. tol <= 0 -> sqrt(max(m,n)) *
 * 2^-24. Level-0 matrices iterate in fp32 (FFMA). Gram-path matrices iterate, by default, on an fp64
 * working copy with the FP64 DMMA contractions (sm_100a has no full-precision fp32 MMA: DMMA is
 * fp64-only, TF32 keeps 10 mantissa bits; an FFMA contraction needs 8x the issue slots of DMMA per
 * flop while the FP32 pipe is only 2x the FP64 one, so this is the fastest route) and are rounded to
 * fp32 at finalisation; opts->f32_compute = 1 selects the all-fp32 Gram path (FFMA Gram / update, fp32
 * EVD and Newton-Schulz on an fp32 working copy). Accuracy targets (north_star): sigma 1e-5, residual
 * 1e-5, orthogonality 1e-4, all relative. */
WCSVD_API int wcsvd_batched_f32(int batch, const int* m, const int* n, const float* const* A, const int* lda,
                                float* const* S, float* const* U, float* const* V, float tol, int max_sweeps,
                                wcsvd_stream_t stream);
WCSVD_API int wcsvd_batched_f32_ex(int batch, const int* m, const int* n, const float* const* A,
                                   const int* lda, float* const* S, float* const* U, float* const* V,
                                   float tol, int max_sweeps, wcsvd_stream_t stream, const wcsvd_opts* opts);

/* wcsvd_batched_host -- the same factorisation with HOST buffers (the end-to-end call: host -> device
 * copies, the iteration and device -> host copies all inside).
 *   A[b], S[b], U[b], V[b]: HOST pointers (column-major, lda / ldu / ldv as in wcsvd_batched). Page-locked
 *     memory gives full copy/compute overlap; pageable memory is accepted (the copies then block the
 *     calling thread per chunk and overlap less).
 *   U, V: NULL, or an array of non-NULL pointers for every matrix (-7 if some entries are NULL).
 *   opts: as wcsvd_batched_ex, except that opts->info is a HOST int[batch]; workspace is ignored.
 * Pipeline: the batch is cut into contiguous chunks of about equal estimated cost -- a uniform Level-0
 * batch into ~500-matrix chunks (<= 32), a uniform Gram-path batch into min(16, batch / 128) chunks (at
 * least 1), a mixed-size batch into 3 chunks when it has >= 300 matrices (else 1). Chunk c is copied in
 * (stream 1), factored on one of two compute streams, and copied out (stream 2) while later chunks are
 * copied in / factored, through three device staging sets (chunk c's H2D waits for the D2H of chunk
 * c-3); a batch of one chunk is copied in, factored and copied out in order on `stream` (no pipeline
 * streams to set up). Host blocks of consecutive matrices that are adjacent and packed (ld = rows) move as one copy
 * (per matrix if the runtime refuses a merged range).
 * Zero-copy route: when EVERY host buffer is page-locked and mapped into the device address space
 * (cudaHostAlloc / cudaMallocHost / torch pin_memory under UVA) and the batch is compute-heavy (estimated
 * 10-sweep textbook flops >= 1200 per byte of A + S + U + V; e.g. C5's mixed 32..1024 sizes), the
 * kernels read A and write S, U, V in host memory directly: the transfers happen inside the kernels
 * (each input read once at stage-in, each output written once at finalisation) and overlap other
 * matrices' sweeps, with no staging and no chunk boundaries (measured C5 e2e 957 -> 1032 matrices/s).
 * Smaller / Level-0-sized batches keep the staged pipeline (zero-copy measured slower there).
 * Ordered after prior work on `stream`; SYNCHRONOUS: returns when every output is in host memory.
 * Results are bitwise those of wcsvd_batched on the same inputs (per-matrix determinism).
 * Errors: the argument checks of wcsvd_batched, opts fields and per-matrix plans included (returned
 * before anything is allocated or enqueued); ENOMEM if the staging cannot be allocated; ECUDA on a
 * failed copy or launch. */
WCSVD_API int wcsvd_batched_host(int batch, const int* m, const int* n, const double* const* A, const int* lda,
                                 double* const* S, double* const* U, double* const* V, double tol,
                                 int max_sweeps, wcsvd_stream_t stream, const wcsvd_opts* opts);

/* Bytes of device workspace wcsvd_batched_ex needs for this batch with default options (planner
 * tailoring; the slot pools are sized from the current device's SM count, 148 if no device is
 * visible). 0 for an invalid batch. */
WCSVD_API size_t wcsvd_workspace_size(int batch, const int* m, const int* n);

/* wcsvd_etkf_analysis -- the data-assimilation consumer of the SVD (§V.F:
 * one SVD per grid point of an ocean model, batched; the paper's DA codes are ensemble Kalman filters,
 * refs [36]-[38] PAPER.md:538-541). Reading R-DA: the ETKF ensemble-space analysis.
 * Per grid point b, with the scaled observation-space ensemble perturbations Y_b (m x n: m obs,
 * n members) = U diag(S) V^T as returned by wcsvd_batched, and the scaled innovation d_b (m):
 *   wbar = (I_n + Y^T Y)^-1 Y^T d = V diag(s / (1 + s^2)) U^T d             (n)
 *   T    = (I_n + Y^T Y)^-1/2     = I_n + V diag((1 + s^2)^-1/2 - 1) V^T      (n x n, symmetric)
 * so that the analysis ensemble is X_a = xbar_b 1^T + X_b' (wbar 1^T + T) (unscaled: see DESIGN.md).
 *  m, n        host [batch], 1..1024.                                                     (2, 3)
 *  S, U, V     host [batch] of DEVICE pointers: S k = min(m,n); U m x k (ld m); V n x k (ld n),
 *              column-major -- exactly wcsvd_batched's outputs for Y_b.                   (4-6)
 *  d           host [batch] of DEVICE pointers to m doubles.                               (7)
 *  wbar, T     host [batch] of DEVICE output pointers: n doubles; n x n column-major (ld n). (8, 9)
 * Asynchronous on `stream`; negative codes (argument index / ENOTSUP / ENOMEM / ECUDA) synchronous,
 * nothing enqueued on an argument error. Deterministic (fixed-order sums, FP64 DMMA tiles). */
WCSVD_API int wcsvd_etkf_analysis(int batch, const int* m, const int* n, const double* const* S,
                                  const double* const* U, const double* const* V, const double* const* d,
                                  double* const* wbar, double* const* T, wcsvd_stream_t stream);

/* Release the cached blocks of the library's workspace pool on the current device (after pending
 * calls complete). Returns WCSVD_OK or WCSVD_ECUDA. */
WCSVD_API int wcsvd_trim_workspace(void);

/* Static string for a status code. */
WCSVD_API const char* wcsvd_status_string(int status);

/* ---- Host-only planner introspection (no CUDA call; used by tests and the multi-GPU split) ---- */

/* The per-matrix plan, a pure function of (m, n) (and an optional forced path / width). */
typedef struct {
  int m, n;            /* input sizes */
  int M, N;            /* working orientation, M = max(m,n) >= N = min(m,n) */
  int swapped;         /* 1 if m < n (the iteration runs on A^T) */
  int path;            /* WCSVD_PATH_L0 / _GRAM / _WCYCLE */
  int n_pad;           /* padded column count: a multiple of 2w (Level >= 1) or the L0 tile width */
  int m_pad;           /* padded row count (multiple of 8) of the Level >= 1 working copy */
  int w;               /* Level-1 block width (0 for L0) */
  int w2;              /* Level-2 block width (W-cycle path), else 0 */
  int variant;         /* kernel variant id (L0 template instance) */
  double cost;         /* estimated flops per sweep, F_tb(M, N) = N(N-1)/2 (8M + 6N) */
} wcsvd_plan_t;

/* Fill *out with the plan for one m x n matrix. Returns WCSVD_OK, -1/-2 for bad m/n, or
 * WCSVD_ENOTSUP. force_path / force_w as in wcsvd_opts (0 = planner). */
WCSVD_API int wcsvd_plan(int m, int n, int force_path, int force_w, wcsvd_plan_t* out);

/* The round-robin (circle-method) schedule used at every level.
 * For `np` indices (even, >= 2) at step `step` (0 <= step < np-1), writes the np/2 disjoint pairs
 * as pairs[2p], pairs[2p+1] (original indices, pairs[2p] < pairs[2p+1]). Returns 0 or -1. */
WCSVD_API int wcsvd_round_robin(int np, int step, int* pairs);

/* Library build identification, e.g. "wcsvd 0.1 sm_100a". */
WCSVD_API const char* wcsvd_version(void);

#ifdef __cplusplus
}
#endif
#endif /* WCSVD_H_ */
