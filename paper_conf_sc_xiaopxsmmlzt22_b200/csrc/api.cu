// api.cu -- the C-ABI (include/wcsvd.h): argument validation, the per-matrix planner (the W-cycle
// level filters), workspace, descriptor upload and kernel launches.
// Host code only; every numerical step runs in the CUDA kernels of this directory.
#include <cuda_runtime.h>

#include <algorithm>
#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <cstdint>
#include <cstring>
#include <mutex>
#include <unordered_map>
#include <vector>

#include "common.cuh"
#include "kernels.h"
#include "plan_table.h"
#include "wcsvd.h"

namespace wcsvd {
namespace {

constexpr int kMaxDim = 1024;
constexpr int kHostSets = 4;         // max device staging sets of the host-buffer pipeline
constexpr int kHostSetsDefault = 3;
// host API: zero-copy route above this estimated flop / byte of I/O (10 sweeps x F_tb over A + S + U + V
// bytes). Measured e2e (B200, matrices/s, staged pipeline vs zero-copy): C5 (1648 flop/B) 956 vs 1032;
// C3 (743) 8983 vs 8022; C4 (327) 11481 vs 9543; C2 (183) 487k vs 144k.
constexpr double kZeroCopyFlopPerByte = 1200.0;

double f_tb(int M, int N) { return 0.5 * N * (N - 1.0) * (8.0 * M + 6.0 * N); }

// Level-0 variant for an M x N (M >= N) matrix, or 0 if it does not fit one CTA's registers.
// Limits follow from <= 256 threads x 255 registers per CTA (l0_jacobi.cu launch_l0 table):
// threads = (ceil(M/R) + NP/R) * G.
int l0_variant(int M, int N) {
  if (N <= 8) return (M / 8 + 2) * 1 <= 256 ? kL0_8 : 0;
  if (N <= 16) return ((M + 7) / 8 + 2) * 2 <= 256 ? kL0_16 : 0;
  if (N <= 32) {
    if (M <= 48) return kL0_32s;
    return ((M + 3) / 4 + 8) * 2 <= 256 ? kL0_32 : 0;
  }
  if (N <= 48) return ((M + 1) / 2 + 24) * 2 <= 256 ? kL0_48 : 0;
  if (N <= 64) return ((M + 7) / 8 + 8) * 8 <= 256 ? kL0_64 : 0;  // G = 8, R = 8
  return 0;
}

// Two-phase Level-0 variant (l0_tp.cu), or 0: X and V_x time-share the registers of one CTA.
int l0tp_variant(int M, int N) {
#ifdef WCSVD_NO_TP
  return 0;  // experiments: fused Level-0 kernel only
#endif
  if (N > 16 && N <= 32 && M > 48 && M <= kTP32MaxM) return kTP32;  // M <= 48: fused kL0_32s (latency)
  if (N > 48 && N <= 64 && M <= kTP64MaxM) return kTP64;
  return 0;
}

// Measured plan table (plan_table.h, tools/autotune.py + tools/gen_plan_table.py): the
// entry nearest to (M, N) in (log N, log M/N), restricted to entries on the same side of the Level-0
// fit (a matrix that fits one CTA is compared with measured shapes that also fit, and vice versa).
const PlanEntry* plan_lookup(int M, int N, bool l0fit) {
  // the table's coordinates and Level-0 fit, computed once (immutable after initialisation)
  struct Coord { double ln, la; bool fit; };
  static const std::vector<Coord> coords = [] {
    std::vector<Coord> c(kPlanTableSize);
    for (int i = 0; i < kPlanTableSize; ++i) {
      const PlanEntry& e = kPlanTable[i];
      c[i] = {std::log((double)e.N), std::log((double)e.M / e.N),
              (l0tp_variant(e.M, e.N) ? 1 : l0_variant(e.M, e.N)) != 0};
    }
    return c;
  }();
  const PlanEntry* best = nullptr;
  double bd = 0;
  const double ln = std::log((double)N), la = std::log((double)M / N);
  for (int i = 0; i < kPlanTableSize; ++i) {
    if (coords[i].fit != l0fit) continue;
    const double dn = coords[i].ln - ln, da = coords[i].la - la;
    const double dd = dn * dn + da * da;
    if (!best || dd < bd) { best = &kPlanTable[i]; bd = dd; }
  }
  return best;
}

int plan_one(int m, int n, int force_path, int force_w, wcsvd_plan_t* p) {
  std::memset(p, 0, sizeof(*p));
  p->m = m;
  p->n = n;
  p->swapped = (m < n) ? 1 : 0;  // iterate on A^T when m < n
  p->M = std::max(m, n);
  p->N = std::min(m, n);
  p->cost = f_tb(p->M, p->N);
  const int tp = l0tp_variant(p->M, p->N);
  const int v = tp ? tp : l0_variant(p->M, p->N);
  // Alg 2 l.2-14 level choice with the B200 measurements deciding among the
  // paths that apply: Level 0 only if the matrix fits one CTA AND the nearest measured shape ran
  // fastest on Level 0; the Gram-path EVD width and the W-cycle from the same table.
  const PlanEntry* pe = (force_path == 0 && force_w == 0) ? plan_lookup(p->M, p->N, v != 0) : nullptr;
  const bool take_l0 = v && (force_path == WCSVD_PATH_L0 || (force_path == 0 && (!pe || pe->path == WCSVD_PATH_L0)));
  if (take_l0) {
    p->path = WCSVD_PATH_L0;
    p->variant = v;
    static const int np_of[] = {0, 8, 16, 32, 32, 48, 64, 32, 64};
    p->n_pad = np_of[v];
    p->m_pad = p->M;
    return WCSVD_OK;
  }
  if (force_path == WCSVD_PATH_L0) return WCSVD_ENOTSUP;
  // Alg 2 l.5-11: Level 1, column blocks of width w; the pair Gram's EVD runs on-chip.
  int w = pe ? (pe->path == WCSVD_PATH_L0 ? pe->wg : pe->w) : ((p->N <= 96) ? 8 : 16);
  if (force_w == 8 || force_w == 16) w = force_w;
  else if (force_w != 0) return WCSVD_ENOTSUP;
  if (force_path == WCSVD_PATH_PANEL || (pe && pe->path == WCSVD_PATH_PANEL)) {
    // Alg 2 l.8-9, group (i): J from the SVD of the pair panel (l1_gram.cu evd_fast32); w = 16
    if (force_w == 8) return WCSVD_ENOTSUP;
    p->path = WCSVD_PATH_PANEL;
    p->w = 16;
    p->n_pad = (p->N + 31) / 32 * 32;
    p->m_pad = (p->M + 15) / 16 * 16;
    p->variant = (p->n_pad / 32 >= 8) ? kL1_32x8 : kL1_32x4;
    return WCSVD_OK;
  }
  if (force_path == WCSVD_PATH_WCYCLE || (pe && pe->path == WCSVD_PATH_WCYCLE)) {
    // Alg 2 l.12-14: w1 = 64 super-blocks recurse to Level 2 with w2 = w (EVD width 2 w2).
    p->path = WCSVD_PATH_WCYCLE;
    p->w = 64;
    p->w2 = w;
    p->n_pad = (p->N + 127) / 128 * 128;
    p->m_pad = (p->M + 15) / 16 * 16;
    p->variant = (w == 8) ? kL1_16x4 : kL1_32x8;
    return WCSVD_OK;
  }
  p->path = WCSVD_PATH_GRAM;
  p->w = w;
  p->n_pad = (p->N + 2 * w - 1) / (2 * w) * (2 * w);
  p->m_pad = (p->M + 15) / 16 * 16;
  const int pairs = p->n_pad / w / 2;
  p->variant = (w == 8) ? kL1_16x4 : (pairs >= 8 ? kL1_32x8 : kL1_32x4);
  static const int env_nw = [] {  // experiments only: WCSVD_L1_NW=4 / 8 forces the 2w = 32 CTA width
    const char* e = std::getenv("WCSVD_L1_NW");
    return e ? std::atoi(e) : 0;
  }();
  if (w == 16 && env_nw == 4) p->variant = kL1_32x4;
  if (w == 16 && env_nw == 8) p->variant = kL1_32x8;
  return WCSVD_OK;
}

// Doubles of one workspace slot for a matrix with plan p: the Level >= 1 working copy W (m_pad x
// n_pad) and V (n_pad x n_pad), or the Level-0 two-phase park buffer; 0 if the path needs none.
size_t slot_doubles(const wcsvd_plan_t& p) {
  if (p.path == WCSVD_PATH_L0) return ((l0tp_park_bytes(p.variant, p.M) + 255) & ~size_t(255)) / sizeof(double);
  const size_t b = (size_t)p.m_pad * p.n_pad + (size_t)p.n_pad * p.n_pad;
  return (b + 31) & ~size_t(31);
}

// Warps per CTA and resident CTAs per SM of the Level-1 variants (255 registers / thread, see
// l1_gram.cu launch bounds): the tailoring rule and the slot-pool capacity use them.
int l1_warps(int variant) { return variant == kL1_32x8 ? 8 : 4; }
int resident_per_sm(const wcsvd_plan_t& p) {
  if (p.path == WCSVD_PATH_L0) {
    // two-phase kernels: the slot pool must cover every CTA that can be resident (fp64 or fp32 build)
    const int a = l0tp_occupancy(p.variant, 0, p.M), b = l0tp_occupancy(p.variant, 1, p.M);
    const int r = a > b ? a : b;
    if (r <= 0) cudaGetLastError();  // no device (CPU-side planning): clear the query's error
    return r > 0 ? r : 8;
  }
  static const int env_res4 = [] {  // experiments only: builds with WCSVD_L1_MINB(4) = 3
    const char* e = std::getenv("WCSVD_L1_RES4");
    return e ? std::atoi(e) : 0;
  }();
  if (p.variant == kL1_32x4 && env_res4 > 0) return env_res4;
  return p.variant == kL1_32x8 ? 1 : 2;
}

int device_sms() {
  int dev = 0, sms = 0;
  if (cudaGetDevice(&dev) != cudaSuccess || cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess) {
    cudaGetLastError();
    return 148;  // B200
  }
  return sms;
}

// Tailoring (PAPER.md:228 Challenge 2, §IV.D): CTAs per matrix for the
// flat Gram path. A matrix whose one-CTA time would exceed the whole batch's ideal time on
// the GPU (its cost share c_k / sum c > 1 / (R SMs)) is spread over a cluster of CL CTAs, the
// smallest power of two that brings it under that bound, capped by the pair-level parallelism of a
// round-robin step (ceil(pairs / warps); measured: 8 x 1024^2 in 903 / 455 / 234 / 233 ms on 1 / 2 /
// 4 / 8 CTAs -- the dataflow schedule overlaps steps only a little) and 8.
// A function of the batch's (m, n) multiset only -- it changes scheduling, never arithmetic (Z22).
int choose_cluster(const wcsvd_plan_t& p, double share, int sms) {
  if (p.path != WCSVD_PATH_GRAM) return 1;
  const int nw = l1_warps(p.variant);
  const int pairs = p.n_pad / p.w / 2;
  int cap = 1;
  while (cap < 8 && 2 * cap <= (pairs + nw - 1) / nw) cap *= 2;
  static const double factor = [] {  // experiments only: WCSVD_TAILOR=<f> (default 1; measured C5 at 4 GPUs 776 / 812 / 840 ms for 1 / 2 / 4)
    const char* s = std::getenv("WCSVD_TAILOR");
    return s ? std::atof(s) : 1.0;
  }();
  const double need = factor * resident_per_sm(p) * sms * share;
  int cl = 1;
  while (cl < cap && cl < need) cl *= 2;
  return cl;
}

struct Bucket {
  int path, variant, withv, cluster;
  std::vector<int> members;  // batch indices, largest cost first
  int maxM = 0;
  size_t slot = 0;  // doubles per slot (0: the path needs no workspace)
  int nslots = 0;
  int per_sm = 1;  // slot-pool probe stride per SM (SlotPool::per_sm)
  size_t off_slots = 0, off_busy = 0;  // workspace offsets
};

// Plans, buckets and the workspace layout of one call: a pure function of (m, n, forced options,
// which factors are requested) and of the device's SM count (slot-pool capacity only).
struct CallPlan {
  std::vector<wcsvd_plan_t> plans;
  std::vector<Bucket> buckets;
  size_t off_descs = 0, off_order = 0, off_status = 0, bytes = 0;
};

// tot_cost > 0: the tailoring shares are taken against this total (the host pipeline plans each chunk
// against the whole batch, whose chunks run concurrently), else against this call's own batch.
int make_call_plan(int batch, const int* m, const int* n, int force_path, int force_w, int force_cluster,
                   const std::vector<int>* withv, CallPlan* cp, double tot_cost = 0.0) {
  cp->plans.assign(batch, wcsvd_plan_t{});
  double tot = 0;
  // plan_one is a pure function of (m, n) for fixed options: plan each distinct shape once (a
  // uniform batch of 10,000 matrices otherwise spent ~7 ms of host time in the table search)
  std::unordered_map<uint64_t, int> seen;
  for (int b = 0; b < batch; ++b) {
    const uint64_t key = ((uint64_t)(uint32_t)m[b] << 32) | (uint32_t)n[b];
    auto it = seen.find(key);
    if (it != seen.end()) {
      cp->plans[b] = cp->plans[it->second];
    } else {
      const int rc = plan_one(m[b], n[b], force_path, force_w, &cp->plans[b]);
      if (rc != WCSVD_OK) return rc;
      seen.emplace(key, b);
    }
    tot += cp->plans[b].cost;
  }
  if (tot_cost > 0) tot = tot_cost;
  const int sms = device_sms();
  auto& buckets = cp->buckets;
  buckets.clear();
  for (int b = 0; b < batch; ++b) {
    const wcsvd_plan_t& p = cp->plans[b];
    int cl = force_cluster > 0 ? force_cluster : choose_cluster(p, tot > 0 ? p.cost / tot : 1.0, sms);
    if (p.path != WCSVD_PATH_GRAM) cl = 1;
    // the fused Level-0 kernel is instantiated per "V requested"; every other kernel reads d.withv
    const bool fused_l0 = p.path == WCSVD_PATH_L0 && p.variant != kTP32 && p.variant != kTP64;
    const int wv = (fused_l0 && withv) ? (*withv)[b] : 0;
    Bucket* bk = nullptr;
    for (auto& x : buckets)
      if (x.path == p.path && x.variant == p.variant && x.withv == wv && x.cluster == cl) bk = &x;
    if (!bk) {
      buckets.push_back(Bucket{p.path, p.variant, wv, cl, {}, 0, 0, 0, 0, 0});
      bk = &buckets.back();
    }
    bk->members.push_back(b);
    bk->maxM = std::max(bk->maxM, p.M);
    bk->slot = std::max(bk->slot, slot_doubles(p));
  }
  for (auto& bk : buckets)
    std::stable_sort(bk.members.begin(), bk.members.end(),
                     [&](int x, int y) { return cp->plans[x].cost > cp->plans[y].cost; });
  std::sort(buckets.begin(), buckets.end(), [&](const Bucket& x, const Bucket& y) {
    return cp->plans[x.members[0]].cost > cp->plans[y.members[0]].cost;
  });
  size_t off = 0;
  auto align = [](size_t x) { return (x + 255) & ~size_t(255); };
  cp->off_descs = off;
  off = align(off + sizeof(MatDesc) * (size_t)batch);
  cp->off_order = off;
  off = align(off + sizeof(int) * (size_t)batch);
  cp->off_status = off;
  off = align(off + sizeof(int) * (size_t)batch);
  for (auto& bk : buckets) {
    if (!bk.slot) continue;
    const int cap = std::max(1, (resident_per_sm(cp->plans[bk.members[0]]) * sms + bk.cluster - 1) / bk.cluster);
    bk.nslots = std::min((int)bk.members.size(), cap);
    bk.per_sm = std::max(1, resident_per_sm(cp->plans[bk.members[0]]) / bk.cluster);
    if (std::getenv("WCSVD_SLOTS_ALL")) bk.nslots = (int)bk.members.size();  // experiments: one slot per matrix
    bk.off_busy = off;
    off = align(off + sizeof(int) * (size_t)bk.nslots);
  }
  for (auto& bk : buckets) {
    if (!bk.slot) continue;
    bk.off_slots = off;
    off = align(off + sizeof(double) * bk.slot * (size_t)bk.nslots);
  }
  cp->bytes = off;
  return WCSVD_OK;
}

const char* kStatus[] = {"ok", "invalid argument", "not supported", "CUDA error", "out of memory"};

// The library's own stream-ordered memory pool on `dev` (created once, kept for the process). Freed
// workspace stays cached in it (release threshold = max) so repeated calls do not re-map memory; the
// device's default pool and the caller's allocator are never touched. wcsvd_trim_workspace() releases it.
std::mutex g_pool_mu;
cudaMemPool_t g_pools[64] = {};

cudaError_t lib_pool(cudaMemPool_t* out) {
  int dev = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return e;
  if (dev < 0 || dev >= 64) return cudaErrorInvalidDevice;
  std::lock_guard<std::mutex> lk(g_pool_mu);
  if (!g_pools[dev]) {
    cudaMemPoolProps props;
    std::memset(&props, 0, sizeof(props));
    props.allocType = cudaMemAllocationTypePinned;
    props.location.type = cudaMemLocationTypeDevice;
    props.location.id = dev;
    cudaMemPool_t p;
    e = cudaMemPoolCreate(&p, &props);
    if (e != cudaSuccess) return e;
    uint64_t thr = UINT64_MAX;
    cudaMemPoolSetAttribute(p, cudaMemPoolAttrReleaseThreshold, &thr);
    g_pools[dev] = p;
  }
  *out = g_pools[dev];
  return cudaSuccess;
}

cudaError_t lib_malloc(void** p, size_t bytes, cudaStream_t stream) {
  cudaMemPool_t pool;
  cudaError_t e = lib_pool(&pool);
  if (e != cudaSuccess) return e;
  return cudaMallocFromPoolAsync(p, bytes, pool, stream);
}

// Argument checks shared by every entry point (returned before anything is enqueued).
template <typename TI>
int validate(int batch, const int* m, const int* n, const TI* const* A, const int* lda, TI* const* S, TI* const* U,
             TI* const* V, double tol, const wcsvd_opts* opts) {
  if (batch < 0) return -1;
  if (batch == 0) return WCSVD_OK;
  if (!m) return -2;
  if (!n) return -3;
  if (!A) return -4;
  if (!lda) return -5;
  if (!S) return -6;
  if (opts && opts->struct_size != sizeof(wcsvd_opts)) return -12;
  if (std::isnan(tol)) return -9;
  const int* ldu = opts ? opts->ldu : nullptr;
  const int* ldv = opts ? opts->ldv : nullptr;
  for (int b = 0; b < batch; ++b) {
    if (m[b] < 1) return -2;
    if (n[b] < 1) return -3;
    if (!A[b]) return -4;
    if (lda[b] < m[b]) return -5;
    if (!S[b]) return -6;
    if (ldu && U && U[b] && ldu[b] < m[b]) return -12;
    if (ldv && V && V[b] && ldv[b] < n[b]) return -12;
  }
  for (int b = 0; b < batch; ++b)
    if (m[b] > kMaxDim || n[b] > kMaxDim) return WCSVD_ENOTSUP;
  if (opts) {
    if (opts->pair_warps != 0 && opts->pair_warps != 1) return -12;
    const int c = opts->cluster_ctas;
    if (c != 0 && c != 1 && c != 2 && c != 4 && c != 8) return -12;
    if (opts->f32_compute != 0 && opts->f32_compute != 1) return -12;
    if (opts->force_path < 0 || opts->force_path > WCSVD_PATH_PANEL) return -12;
    if (opts->force_w != 0 && opts->force_w != 8 && opts->force_w != 16) return -12;
    std::unordered_map<uint64_t, int> seen;  // each distinct shape once (plan_one is pure)
    for (int b = 0; b < batch; ++b) {
      if (!seen.emplace(((uint64_t)(uint32_t)m[b] << 32) | (uint32_t)n[b], 0).second) continue;
      wcsvd_plan_t p;
      const int rc = plan_one(m[b], n[b], opts->force_path, opts->force_w, &p);
      if (rc != WCSVD_OK) return rc;
    }
  }
  return WCSVD_OK;
}

}  // namespace
}  // namespace wcsvd

using namespace wcsvd;

template <typename TI>
static int batched_impl(int batch, const int* m, const int* n, const TI* const* A, const int* lda,
                        TI* const* S, TI* const* U, TI* const* V, double tol, int max_sweeps,
                        wcsvd_stream_t stream_, const wcsvd_opts* opts, double tailor_total = 0.0) {
  constexpr bool kF32 = sizeof(TI) == 4;
  const double eps = kF32 ? 5.9604644775390625e-08 : kU53;  // 2^-24 or 2^-53
  cudaStream_t stream = reinterpret_cast<cudaStream_t>(stream_);
  // ---- validation (nothing is enqueued on failure) ----
  const int vr = validate<TI>(batch, m, n, A, lda, S, U, V, tol, opts);
  if (vr != WCSVD_OK || batch == 0) return vr;
  const int* ldu = opts ? opts->ldu : nullptr;
  const int* ldv = opts ? opts->ldv : nullptr;
  const int force_path = opts ? opts->force_path : 0;
  const int force_w = opts ? opts->force_w : 0;
  if (max_sweeps <= 0) max_sweeps = 60;

  // ---- plan (a pure function of (m, n)), tailoring and buckets ----
  // V_x (the square factor) is accumulated only if it is requested: as V when m >= n, as U when
  // m < n (§8(f4) values / U-only mode otherwise; the iteration itself is unchanged).
  std::vector<int> withv(batch);
  for (int b = 0; b < batch; ++b)
    withv[b] = (m[b] < n[b]) ? (U && U[b] ? 1 : 0) : (V && V[b] ? 1 : 0);
  CallPlan cp;
  const int rc0 = make_call_plan(batch, m, n, force_path, force_w, opts ? opts->cluster_ctas : 0, &withv, &cp,
                                 tailor_total);
  // (the fp32 FFMA route, opts->f32_compute = 1, has no PANEL variant: such buckets run fp64-inside)
  if (rc0 != WCSVD_OK) return rc0;
  const auto& plans = cp.plans;
  const auto& buckets = cp.buckets;

  // ---- workspace: descriptors, launch order, status, slot pools ----
  unsigned char* ws = nullptr;
  bool own_ws = false;
  if (opts && opts->workspace) {
    if (opts->workspace_bytes < cp.bytes) return -12;
    ws = static_cast<unsigned char*>(opts->workspace);
  } else {
    if (lib_malloc(reinterpret_cast<void**>(&ws), cp.bytes, stream) != cudaSuccess) {
      cudaGetLastError();
      return WCSVD_ENOMEM;
    }
    own_ws = true;
  }
  MatDesc* d_descs = reinterpret_cast<MatDesc*>(ws + cp.off_descs);
  int* d_order = reinterpret_cast<int*>(ws + cp.off_order);
  int* d_status = reinterpret_cast<int*>(ws + cp.off_status);

  // ---- descriptors (host) -> device ----
  std::vector<MatDesc> h(batch);
  for (int b = 0; b < batch; ++b) {
    const wcsvd_plan_t& p = plans[b];
    MatDesc& d = h[b];
    std::memset(&d, 0, sizeof(d));
    // typed I/O pointers are carried as double* and reinterpreted by the kernels (d.fp32)
    d.A = reinterpret_cast<const double*>(A[b]);
    d.S = reinterpret_cast<double*>(S[b]);
    d.U = U ? reinterpret_cast<double*>(U[b]) : nullptr;
    d.V = V ? reinterpret_cast<double*>(V[b]) : nullptr;
    d.fp32 = kF32 ? 1 : 0;
    d.info = opts ? opts->info : nullptr;
    d.sweeps_inner = opts ? opts->sweeps_inner : nullptr;
    d.m = m[b];
    d.n = n[b];
    d.lda = lda[b];
    d.ldu = ldu ? ldu[b] : m[b];
    d.ldv = ldv ? ldv[b] : n[b];
    d.M = p.M;
    d.N = p.N;
    d.swapped = p.swapped;
    d.m_pad = p.m_pad;
    d.n_pad = p.n_pad;
    d.w = p.w;
    d.w2 = p.w2;
    d.tol = (tol > 0) ? tol : std::sqrt((double)p.M) * eps;
    d.max_sweeps = max_sweeps;
    d.inner_cap = (opts && opts->inner_sweeps > 0) ? opts->inner_sweeps : 1;
    d.inner_cap2 = (opts && opts->wcycle_sweeps > 0) ? opts->wcycle_sweeps : 2;
    d.idx = b;
    d.status = d_status;
    d.withv = withv[b];
  }
  std::vector<int> h_order;
  h_order.reserve(batch);
  std::vector<int> bucket_off;
  size_t busy_lo = cp.bytes, busy_hi = 0;
  for (auto& bk : buckets) {
    bucket_off.push_back((int)h_order.size());
    h_order.insert(h_order.end(), bk.members.begin(), bk.members.end());
    if (bk.slot) {
      busy_lo = std::min(busy_lo, bk.off_busy);
      busy_hi = std::max(busy_hi, bk.off_busy + sizeof(int) * (size_t)bk.nslots);
    }
  }
  cudaError_t e = cudaMemcpyAsync(d_descs, h.data(), sizeof(MatDesc) * batch, cudaMemcpyHostToDevice, stream);
  if (e == cudaSuccess)
    e = cudaMemcpyAsync(d_order, h_order.data(), sizeof(int) * batch, cudaMemcpyHostToDevice, stream);
  if (e == cudaSuccess && busy_hi > busy_lo) e = cudaMemsetAsync(ws + busy_lo, 0, busy_hi - busy_lo, stream);

  // ---- launches ----
  // One launch per plan bucket (largest first). With several buckets (mixed sizes) each runs on its
  // own stream forked from `stream` so small buckets fill the SMs that large ones leave idle; all
  // are joined back into `stream` before the completion pass. Per-matrix results do not depend on
  // this concurrency, on the slot a matrix gets, or on its CTA count.
  const int nbk = (int)buckets.size();
  std::vector<cudaStream_t> side(nbk > 1 ? nbk : 0, nullptr);
  std::vector<cudaEvent_t> done(side.size(), nullptr);
  cudaEvent_t fork = nullptr;
  if (nbk > 1 && e == cudaSuccess) {
    e = cudaEventCreateWithFlags(&fork, cudaEventDisableTiming);
    if (e == cudaSuccess) e = cudaEventRecord(fork, stream);
    for (int i = 0; i < nbk && e == cudaSuccess; ++i) {
      e = cudaStreamCreateWithFlags(&side[i], cudaStreamNonBlocking);
      if (e == cudaSuccess) e = cudaEventCreateWithFlags(&done[i], cudaEventDisableTiming);
      if (e == cudaSuccess) e = cudaStreamWaitEvent(side[i], fork, 0);
    }
  }
  for (int i = 0; i < nbk && e == cudaSuccess; ++i) {
    const Bucket& bk = buckets[i];
    const int cnt = (int)bk.members.size();
    cudaStream_t st = (nbk > 1) ? side[i] : stream;
    SlotPool pool{nullptr, 0, nullptr, 0, 1};
    if (bk.slot) pool = SlotPool{reinterpret_cast<double*>(ws + bk.off_slots), bk.slot,
                                 reinterpret_cast<int*>(ws + bk.off_busy), bk.nslots, bk.per_sm};
    if (bk.path == WCSVD_PATH_L0 && (bk.variant == kTP32 || bk.variant == kTP64))
      e = launch_l0tp(bk.variant, kF32 ? 1 : 0, d_descs, d_order + bucket_off[i], cnt, bk.maxM, pool, st);
    else if (bk.path == WCSVD_PATH_L0)
      e = launch_l0(bk.variant, bk.withv, kF32 ? 1 : 0, d_descs, d_order + bucket_off[i], cnt, bk.maxM, st);
    else
      e = launch_l1(bk.variant, bk.path == WCSVD_PATH_WCYCLE ? 1 : (bk.path == WCSVD_PATH_PANEL ? 2 : 0), kF32 ? 1 : 0,
                    (opts && opts->f32_compute && bk.path != WCSVD_PATH_PANEL) ? 1 : 0,
                    d_descs, d_order + bucket_off[i], cnt, bk.cluster, pool, st);
    if (e == cudaSuccess && nbk > 1) e = cudaEventRecord(done[i], st);
  }
  for (int i = 0; i < (int)side.size(); ++i) {
    if (e == cudaSuccess && done[i]) e = cudaStreamWaitEvent(stream, done[i], 0);
  }
  for (int i = 0; i < (int)side.size(); ++i) {
    if (done[i]) cudaEventDestroy(done[i]);
    if (side[i]) cudaStreamDestroy(side[i]);  // released once its work completes
  }
  if (fork) cudaEventDestroy(fork);
  if (e == cudaSuccess) e = launch_complete(kF32 ? 1 : 0, d_descs, batch, stream);
  if (own_ws) cudaFreeAsync(ws, stream);
  if (e != cudaSuccess) {
    if (std::getenv("WCSVD_DEBUG")) std::fprintf(stderr, "wcsvd: %s\n", cudaGetErrorString(e));
    cudaGetLastError();
    return WCSVD_ECUDA;
  }
  return WCSVD_OK;
}

// ---- Host-buffer entry point: chunked three-stage pipeline (H2D / kernels / D2H) ----
// The batch is cut into contiguous chunks; chunk c is copied in on `s_in`, factored by batched_impl
// on its own compute stream (two alternate, so a chunk's first wave starts while the previous one
// drains), and copied out on `s_out`, with two device staging sets: copies overlap the iteration.
// Host ranges that are contiguous (consecutive matrices packed back to back, ld = rows) move as one
// copy per chunk and array; anything else falls back to one 2-D copy per matrix.
namespace {

struct HostRun {
  size_t dst_off;   // element offset in the device staging array
  const void* src;  // host base (H2D) / destination (D2H)
  size_t elems;     // total elements of a packed run (ld == rows), else 0
  int rows, cols, ld;
  int b0, nb;       // the matrices of the run (per-matrix fallback)
};

// True if the whole batch of this array is one packed block in host memory (a [B, ...] array): only
// then are adjacent matrices merged into one copy (separately allocated page-locked buffers that happen
// to be adjacent may not be spanned by one copy).
template <typename Ptr>
bool whole_adjacent(int batch, Ptr host, const int* rows, const int* cols, const int* ld) {
  for (int b = 1; b < batch; ++b)
    if (ld[b - 1] != rows[b - 1] ||
        reinterpret_cast<const double*>(host[b - 1]) + (size_t)rows[b - 1] * cols[b - 1] != reinterpret_cast<const double*>(host[b]))
      return false;
  return ld[0] == rows[0];
}

// Group matrices [b0, b1) into copy runs: consecutive packed matrices whose host blocks are adjacent
// (when `merge`), else one run per matrix.
template <typename Ptr>
std::vector<HostRun> host_runs(int b0, int b1, const std::vector<size_t>& off, Ptr host, const int* rows,
                               const int* cols, const int* ld, bool merge) {
  std::vector<HostRun> runs;
  for (int b = b0; b < b1; ++b) {
    const size_t el = (size_t)rows[b] * cols[b];
    const bool packed = ld[b] == rows[b];
    if (merge && !runs.empty() && packed && runs.back().elems &&
        reinterpret_cast<const double*>(runs.back().src) + runs.back().elems == reinterpret_cast<const double*>(host[b]) &&
        runs.back().dst_off + runs.back().elems == off[b]) {
      runs.back().elems += el;
      ++runs.back().nb;
      continue;
    }
    runs.push_back(HostRun{off[b], host[b], packed ? el : 0, rows[b], cols[b], ld[b], b, 1});
  }
  return runs;
}

// One run of host <-> device copies. Host blocks that are adjacent in the address space may still
// belong to different page-locked allocations (a copy may not span those: cudaErrorInvalidValue), so a
// merged run that is refused is redone matrix by matrix.
template <typename Ptr>
cudaError_t copy_run(const HostRun& r, bool h2d, double* dev, const std::vector<size_t>& off, Ptr host,
                     const int* rows, const int* cols, const int* ld, cudaStream_t st) {
  const size_t es = sizeof(double);
  auto one = [&](size_t doff, const void* h, size_t elems, int rr, int cc, int l) {
    if (elems)
      return h2d ? cudaMemcpyAsync(dev + doff, h, elems * es, cudaMemcpyHostToDevice, st)
                 : cudaMemcpyAsync(const_cast<void*>(h), dev + doff, elems * es, cudaMemcpyDeviceToHost, st);
    return h2d ? cudaMemcpy2DAsync(dev + doff, (size_t)rr * es, h, (size_t)l * es, (size_t)rr * es, cc,
                                   cudaMemcpyHostToDevice, st)
               : cudaMemcpy2DAsync(const_cast<void*>(h), (size_t)l * es, dev + doff, (size_t)rr * es,
                                   (size_t)rr * es, cc, cudaMemcpyDeviceToHost, st);
  };
  cudaError_t e = one(r.dst_off, r.src, r.elems, r.rows, r.cols, r.ld);
  if (e == cudaErrorInvalidValue && r.nb > 1) {
    cudaGetLastError();
    e = cudaSuccess;
    for (int b = r.b0; b < r.b0 + r.nb && e == cudaSuccess; ++b)
      e = one(off[b], host[b], (size_t)rows[b] * cols[b], rows[b], cols[b], ld[b]);
  }
  return e;
}

}  // namespace

// The host pipeline's streams and events, created once per host thread and device and reused by every
// later call (creating 4 streams and ~12 events cost ~0.4 ms per call -- as much as C1's kernels). The
// API is synchronous, so a thread's calls never overlap and every call drains these streams before it
// returns; they live as long as the thread (never destroyed, like a library handle).
struct HostPipeline {
  bool ok = false;
  cudaStream_t s_in = nullptr, s_out = nullptr, s_cp[2] = {nullptr, nullptr};
  cudaEvent_t ev_start = nullptr, ev_in[kHostSets] = {}, ev_cp[kHostSets] = {}, ev_out[kHostSets] = {};
  cudaEvent_t ev_join[4] = {};
};
static HostPipeline* host_pipeline() {
  constexpr int kMaxDev = 16;
  thread_local HostPipeline cache[kMaxDev];
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= kMaxDev) {
    cudaGetLastError();
    return nullptr;
  }
  HostPipeline& h = cache[dev];
  if (h.ok) return &h;
  cudaError_t e = cudaStreamCreateWithFlags(&h.s_in, cudaStreamNonBlocking);
  if (e == cudaSuccess) e = cudaStreamCreateWithFlags(&h.s_out, cudaStreamNonBlocking);
  for (int i = 0; i < 2 && e == cudaSuccess; ++i) e = cudaStreamCreateWithFlags(&h.s_cp[i], cudaStreamNonBlocking);
  for (int i = 0; i < kHostSets && e == cudaSuccess; ++i) {
    e = cudaEventCreateWithFlags(&h.ev_in[i], cudaEventDisableTiming);
    if (e == cudaSuccess) e = cudaEventCreateWithFlags(&h.ev_cp[i], cudaEventDisableTiming);
    if (e == cudaSuccess) e = cudaEventCreateWithFlags(&h.ev_out[i], cudaEventDisableTiming);
  }
  for (int i = 0; i < 4 && e == cudaSuccess; ++i) e = cudaEventCreateWithFlags(&h.ev_join[i], cudaEventDisableTiming);
  if (e == cudaSuccess) e = cudaEventCreateWithFlags(&h.ev_start, cudaEventDisableTiming);
  if (e != cudaSuccess) {
    cudaGetLastError();
    return nullptr;  // the caller reports ECUDA; the next call retries the creation
  }
  h.ok = true;
  return &h;
}

// Device-visible alias of a host pointer if it is page-locked and mapped (cudaHostAlloc / torch
// pin_memory under UVA), else nullptr (pageable memory: the staged pipeline is used).
static void* mapped_alias(const void* p) {
  if (!p) return nullptr;
  cudaPointerAttributes at;
  if (cudaPointerGetAttributes(&at, p) != cudaSuccess) {
    cudaGetLastError();
    return nullptr;
  }
  return (at.type == cudaMemoryTypeHost && at.devicePointer) ? at.devicePointer : nullptr;
}

// Zero-copy route of wcsvd_batched_host: every host buffer is mapped, so the kernels
// read A and write S, U, V in host memory themselves -- the host <-> device transfers happen inside
// the kernels (stage-in reads A once, finalisation writes each output once) and overlap the other
// CTAs' sweeps, with no staging copies and no chunk boundaries. Returns 1 if the route does not apply.
static int batched_host_zero_copy(int batch, const int* m, const int* n, const double* const* A, const int* lda,
                                  double* const* S, double* const* U, double* const* V, double tol, int max_sweeps,
                                  cudaStream_t stream, const wcsvd_opts* opts) {
  // policy: compute-heavy batches only (estimated flops per byte of I/O; the Level-0-sized ones keep
  // the copy-engine pipeline, whose transfers already hide behind their short kernels). Env
  // WCSVD_HOST_ZEROCOPY=0/1 forces the choice (experiments).
  const char* env = std::getenv("WCSVD_HOST_ZEROCOPY");
  if (env && std::atoi(env) == 0) return 1;
  double fl = 0, by = 0;
  for (int b = 0; b < batch; ++b) {
    const int M = std::max(m[b], n[b]), N = std::min(m[b], n[b]);
    fl += 10.0 * f_tb(M, N);
    by += 8.0 * ((double)m[b] * n[b] + (double)N * (m[b] + n[b] + 1));
  }
  if (!(env && std::atoi(env) == 1) && fl < kZeroCopyFlopPerByte * by) return 1;
  std::vector<const double*> pA(batch);
  std::vector<double*> pS(batch), pU(U ? batch : 0), pV(V ? batch : 0);
  for (int b = 0; b < batch; ++b) {
    pA[b] = static_cast<const double*>(mapped_alias(A[b]));
    pS[b] = static_cast<double*>(mapped_alias(S[b]));
    if (!pA[b] || !pS[b]) return 1;
    if (U && !(pU[b] = static_cast<double*>(mapped_alias(U[b])))) return 1;
    if (V && !(pV[b] = static_cast<double*>(mapped_alias(V[b])))) return 1;
  }
  int* h_info = opts ? opts->info : nullptr;  // HOST int[batch] (may be pageable)
  int* d_info = nullptr;
  if (h_info && lib_malloc(reinterpret_cast<void**>(&d_info), sizeof(int) * (size_t)batch, stream) != cudaSuccess) {
    cudaGetLastError();
    return WCSVD_ENOMEM;
  }
  wcsvd_opts o;
  std::memset(&o, 0, sizeof(o));
  o.struct_size = sizeof(o);
  o.info = d_info;
  if (opts) {
    o.ldu = opts->ldu;
    o.ldv = opts->ldv;
    o.force_path = opts->force_path;
    o.force_w = opts->force_w;
    o.wcycle_sweeps = opts->wcycle_sweeps;
    o.inner_sweeps = opts->inner_sweeps;
    o.pair_warps = opts->pair_warps;
    o.cluster_ctas = opts->cluster_ctas;
    o.f32_compute = opts->f32_compute;
  }
  const int rc = batched_impl<double>(batch, m, n, pA.data(), lda, pS.data(), U ? pU.data() : nullptr,
                                      V ? pV.data() : nullptr, tol, max_sweeps,
                                      reinterpret_cast<wcsvd_stream_t>(stream), &o);
  cudaError_t e = cudaSuccess;
  if (rc == WCSVD_OK && h_info) e = cudaMemcpyAsync(h_info, d_info, sizeof(int) * (size_t)batch, cudaMemcpyDeviceToHost, stream);
  if (d_info) cudaFreeAsync(d_info, stream);
  const cudaError_t es2 = cudaStreamSynchronize(stream);  // synchronous API: outputs are in host memory
  if (rc != WCSVD_OK) return rc;
  if (e != cudaSuccess || es2 != cudaSuccess) {
    cudaGetLastError();
    return WCSVD_ECUDA;
  }
  return WCSVD_OK;
}

static int batched_host_impl(int batch, const int* m, const int* n, const double* const* A, const int* lda,
                             double* const* S, double* const* U, double* const* V, double tol, int max_sweeps,
                             wcsvd_stream_t stream_, const wcsvd_opts* opts) {
  cudaStream_t stream = reinterpret_cast<cudaStream_t>(stream_);
  // every argument (opts fields and per-matrix plans included) is checked before anything is enqueued
  const int vr = validate<double>(batch, m, n, A, lda, S, U, V, tol, opts);
  if (vr != WCSVD_OK || batch == 0) return vr;
  const int* ldu = opts ? opts->ldu : nullptr;
  const int* ldv = opts ? opts->ldv : nullptr;
  const bool wantU = U != nullptr, wantV = V != nullptr;
  for (int b = 0; b < batch && (wantU || wantV); ++b)
    if ((wantU && !U[b]) || (wantV && !V[b])) return -7;  // host API: a factor is requested for all or none
  {
    const int zc = batched_host_zero_copy(batch, m, n, A, lda, S, U, V, tol, max_sweeps, stream, opts);
    if (zc != 1) return zc;
  }

  // device staging offsets (packed per matrix, in batch order)
  std::vector<size_t> oA(batch), oS(batch), oU(batch), oV(batch);
  std::vector<int> kk(batch), ldu_v(batch), ldv_v(batch);
  // chunks: contiguous index ranges of ~equal textbook cost. A mixed-size batch takes few chunks: its
  // cost-sorted buckets run concurrently only within one call, and the largest matrices of every chunk
  // bound that chunk's duration (two staging sets: C5 e2e 776 with 8 chunks vs 891 with one).
  bool uniform = true;
  for (int b = 1; b < batch && uniform; ++b) uniform = (m[b] == m[0] && n[b] == n[0]);
  // chunk count measured on B200: Level 0 (C2, 10,000 x 64^2) 1/6/12/16/20/24/32 chunks -> 36.4/28.9/
  // 25.6/28.8/23.2/25.2/29.8 ms, i.e. best near 500 matrices per chunk (just under one resident wave of
  // 4 CTAs x 148 SMs, two chunks in flight); Gram path (C3 / C4) 8 chunks (C3 4/6/8/12 -> 262/263/250/
  // 268 ms, C4 1/6/8/12 -> 516/421/413/457 ms) with two staging sets; with three (r01g, e2e matrices/s):
  // C2 20 chunks 424k (2 sets) / 465k (3) / 443k (4), 32 chunks 420k; C3 8 / 16 chunks 8455 / 8467;
  // C4 8 / 16 chunks 9804 / 10634 -> Gram path 16 chunks
  // mixed batches: 3 equal-cost chunks when large (C5, three staging sets, r01i: 1/2/3/4/6 chunks -> e2e
  // 892/906/927/745/620 matrices/s; beyond 3 every chunk is bounded by its own largest matrices)
  // Gram path: 16 chunks at C3 / C4 sizes, fewer for small batches (~128 matrices per chunk at least,
  // so a chunk still fills the GPU; a small batch is one chunk).
  int nch = batch >= 300 ? 3 : 1;
  if (uniform) {
    wcsvd_plan_t p0;
    const bool l0 = plan_one(m[0], n[0], opts ? opts->force_path : 0, opts ? opts->force_w : 0, &p0) == WCSVD_OK &&
                    p0.path == WCSVD_PATH_L0;
    const int want = l0 ? std::min(32, (batch + 499) / 500) : std::min(16, std::max(1, batch / 128));
    nch = std::max(1, std::min(batch, want));
  }
  if (const char* env = std::getenv("WCSVD_HOST_CHUNKS")) nch = std::max(1, std::min(batch, std::atoi(env)));  // experiments
  double tot = 0;
  for (int b = 0; b < batch; ++b) tot += f_tb(std::max(m[b], n[b]), std::min(m[b], n[b]));
  std::vector<int> cb{0};
  double acc = 0;
  for (int b = 0; b < batch; ++b) {
    acc += f_tb(std::max(m[b], n[b]), std::min(m[b], n[b]));
    if ((int)cb.size() < nch && acc >= tot * cb.size() / nch && b + 1 < batch) cb.push_back(b + 1);
  }
  cb.push_back(batch);
  const int C = (int)cb.size() - 1;
  size_t mxA = 0, mxS = 0, mxU = 0, mxV = 0;
  int mxB = 0;
  for (int c = 0; c < C; ++c) {
    size_t a = 0, s = 0, u = 0, v = 0;
    auto up = [](size_t x) { return (x + 31) & ~size_t(31); };  // 256-byte aligned blocks (vector accesses)
    for (int b = cb[c]; b < cb[c + 1]; ++b) {
      kk[b] = std::min(m[b], n[b]);
      oA[b] = a; a = up(a + (size_t)m[b] * n[b]);
      oS[b] = s; s = up(s + kk[b]);
      oU[b] = u; u = up(u + (wantU ? (size_t)m[b] * kk[b] : 0));
      oV[b] = v; v = up(v + (wantV ? (size_t)n[b] * kk[b] : 0));
      ldu_v[b] = ldu ? ldu[b] : m[b];
      ldv_v[b] = ldv ? ldv[b] : n[b];
    }
    mxA = std::max(mxA, a); mxS = std::max(mxS, s); mxU = std::max(mxU, u); mxV = std::max(mxV, v);
    mxB = std::max(mxB, cb[c + 1] - cb[c]);
  }
  const std::vector<int> ones(batch, 1);  // S[b] is a k x 1 block
  const bool mergeA = whole_adjacent(batch, A, m, n, lda);
  const bool mergeS = whole_adjacent(batch, S, kk.data(), ones.data(), kk.data());
  const bool mergeU = wantU && whole_adjacent(batch, U, m, kk.data(), ldu_v.data());
  const bool mergeV = wantV && whole_adjacent(batch, V, n, kk.data(), ldv_v.data());
  const size_t setE = mxA + mxS + mxU + mxV;  // doubles per staging set
  const size_t setB = (setE * sizeof(double) + sizeof(int) * (size_t)mxB + 255) & ~size_t(255);
  // staging sets: chunk c uses set c % NSET, so its H2D waits only for the D2H of chunk c - NSET (with two
  // sets, D2H(c-2) + H2D(c) had to fit inside one chunk's kernel time: bubbles at ~500-matrix chunks)
  int NSET = kHostSetsDefault;
  if (const char* env = std::getenv("WCSVD_HOST_SETS")) NSET = std::max(2, std::min(kHostSets, std::atoi(env)));  // experiments
  NSET = std::min(NSET, std::max(2, C));
  int* h_info = opts ? opts->info : nullptr;  // HOST int[batch] for this entry point
  if (C == 1) {
    // One chunk (small batches, e.g. C1): copy in, factor and copy out in order on the caller's stream
    // -- no pipeline streams or events to create (their setup cost ~0.3 ms per call, as much as C1's
    // kernels), one staging set.
    double* d1 = nullptr;
    if (lib_malloc(reinterpret_cast<void**>(&d1), setB, stream) != cudaSuccess) {
      cudaGetLastError();
      return WCSVD_ENOMEM;
    }
    double* dA = d1;
    double* dS = dA + mxA;
    double* dU = dS + mxS;
    double* dV = dU + mxU;
    int* dI = reinterpret_cast<int*>(dV + mxV);
    cudaError_t x = cudaSuccess;
    for (const HostRun& r : host_runs(0, batch, oA, A, m, n, lda, mergeA)) {
      if (x != cudaSuccess) break;
      x = copy_run(r, true, dA, oA, A, m, n, lda, stream);
    }
    int rc1 = WCSVD_OK;
    if (x == cudaSuccess) {
      std::vector<const double*> pA(batch);
      std::vector<double*> pS(batch), pU(wantU ? batch : 0), pV(wantV ? batch : 0);
      std::vector<int> ld_(batch);
      for (int b = 0; b < batch; ++b) {
        pA[b] = dA + oA[b];
        ld_[b] = m[b];
        pS[b] = dS + oS[b];
        if (wantU) pU[b] = dU + oU[b];
        if (wantV) pV[b] = dV + oV[b];
      }
      wcsvd_opts o;
      std::memset(&o, 0, sizeof(o));
      o.struct_size = sizeof(o);
      o.info = h_info ? dI : nullptr;
      if (opts) {
        o.force_path = opts->force_path;
        o.force_w = opts->force_w;
        o.wcycle_sweeps = opts->wcycle_sweeps;
        o.inner_sweeps = opts->inner_sweeps;
        o.pair_warps = opts->pair_warps;
        o.cluster_ctas = opts->cluster_ctas;
        o.f32_compute = opts->f32_compute;
      }
      rc1 = batched_impl<double>(batch, m, n, pA.data(), ld_.data(), pS.data(), wantU ? pU.data() : nullptr,
                                 wantV ? pV.data() : nullptr, tol, max_sweeps, stream_, &o, tot);
    }
    if (x == cudaSuccess && rc1 == WCSVD_OK) {
      for (const HostRun& r : host_runs(0, batch, oS, S, kk.data(), ones.data(), kk.data(), mergeS)) {
        if (x != cudaSuccess) break;
        x = copy_run(r, false, dS, oS, S, kk.data(), ones.data(), kk.data(), stream);
      }
      if (wantU)
        for (const HostRun& r : host_runs(0, batch, oU, U, m, kk.data(), ldu_v.data(), mergeU)) {
          if (x != cudaSuccess) break;
          x = copy_run(r, false, dU, oU, U, m, kk.data(), ldu_v.data(), stream);
        }
      if (wantV)
        for (const HostRun& r : host_runs(0, batch, oV, V, n, kk.data(), ldv_v.data(), mergeV)) {
          if (x != cudaSuccess) break;
          x = copy_run(r, false, dV, oV, V, n, kk.data(), ldv_v.data(), stream);
        }
      if (h_info && x == cudaSuccess)
        x = cudaMemcpyAsync(h_info, dI, sizeof(int) * (size_t)batch, cudaMemcpyDeviceToHost, stream);
    }
    cudaFreeAsync(d1, stream);
    const cudaError_t es1 = cudaStreamSynchronize(stream);
    if (rc1 != WCSVD_OK) return rc1;
    if (x != cudaSuccess || es1 != cudaSuccess) {
      cudaGetLastError();
      return WCSVD_ECUDA;
    }
    return WCSVD_OK;
  }
  double* dbuf = nullptr;
  if (lib_malloc(reinterpret_cast<void**>(&dbuf), NSET * setB, stream) != cudaSuccess) {
    cudaGetLastError();
    return WCSVD_ENOMEM;
  }
  HostPipeline* hp = host_pipeline();
  if (!hp) {
    cudaFreeAsync(dbuf, stream);
    return WCSVD_ECUDA;
  }
  cudaStream_t s_in = hp->s_in, s_out = hp->s_out, s_cp[2] = {hp->s_cp[0], hp->s_cp[1]};
  cudaEvent_t ev_start = hp->ev_start;
  cudaEvent_t* ev_in = hp->ev_in;
  cudaEvent_t* ev_cp = hp->ev_cp;
  cudaEvent_t* ev_out = hp->ev_out;
  cudaError_t e = cudaEventRecord(ev_start, stream);  // after prior work on `stream` (and the allocation)
  if (e == cudaSuccess) e = cudaStreamWaitEvent(s_in, ev_start, 0);
  if (e == cudaSuccess) e = cudaStreamWaitEvent(s_out, ev_start, 0);
  for (int i = 0; i < 2 && e == cudaSuccess; ++i) e = cudaStreamWaitEvent(s_cp[i], ev_start, 0);
  int rc = WCSVD_OK;
  const size_t es = sizeof(double);
  auto stage = [&](int c, double*& dA, double*& dS, double*& dU, double*& dV, int*& dI) {
    unsigned char* base = reinterpret_cast<unsigned char*>(dbuf) + (c % NSET) * setB;
    dA = reinterpret_cast<double*>(base);
    dS = dA + mxA;
    dU = dS + mxS;
    dV = dU + mxU;
    dI = reinterpret_cast<int*>(dV + mxV);
  };
  auto d2h = [&](int c) -> cudaError_t {
    const int b0 = cb[c], b1 = cb[c + 1], st = c % NSET;
    double *dA, *dS, *dU, *dV;
    int* dI;
    stage(c, dA, dS, dU, dV, dI);
    cudaError_t x = cudaStreamWaitEvent(s_out, ev_cp[st], 0);
    {
      for (const HostRun& r : host_runs(b0, b1, oS, S, kk.data(), ones.data(), kk.data(), mergeS)) {
        if (x != cudaSuccess) break;
        x = copy_run(r, false, dS, oS, S, kk.data(), ones.data(), kk.data(), s_out);
      }
    }
    if (wantU)
      for (const HostRun& r : host_runs(b0, b1, oU, U, m, kk.data(), ldu_v.data(), mergeU)) {
        if (x != cudaSuccess) break;
        x = copy_run(r, false, dU, oU, U, m, kk.data(), ldu_v.data(), s_out);
      }
    if (wantV)
      for (const HostRun& r : host_runs(b0, b1, oV, V, n, kk.data(), ldv_v.data(), mergeV)) {
        if (x != cudaSuccess) break;
        x = copy_run(r, false, dV, oV, V, n, kk.data(), ldv_v.data(), s_out);
      }
    if (h_info && x == cudaSuccess)
      x = cudaMemcpyAsync(h_info + b0, dI, sizeof(int) * (b1 - b0), cudaMemcpyDeviceToHost, s_out);
    if (x == cudaSuccess) x = cudaEventRecord(ev_out[st], s_out);
    return x;
  };
  for (int c = 0; c < C && e == cudaSuccess && rc == WCSVD_OK; ++c) {
    const int b0 = cb[c], b1 = cb[c + 1], cnt = b1 - b0, st = c % NSET, cs = c & 1;
    double *dA, *dS, *dU, *dV;
    int* dI;
    stage(c, dA, dS, dU, dV, dI);
    // H2D into staging set st, once the D2H of chunk c-NSET (same set) has drained it
    if (c >= NSET) e = cudaStreamWaitEvent(s_in, ev_out[st], 0);
    for (const HostRun& r : host_runs(b0, b1, oA, A, m, n, lda, mergeA)) {
      if (e != cudaSuccess) break;
      e = copy_run(r, true, dA, oA, A, m, n, lda, s_in);
    }
    if (e == cudaSuccess) e = cudaEventRecord(ev_in[st], s_in);
    // kernels on compute stream cs
    if (e == cudaSuccess) e = cudaStreamWaitEvent(s_cp[cs], ev_in[st], 0);
    if (e != cudaSuccess) break;
    std::vector<const double*> pA(cnt);
    std::vector<double*> pS(cnt), pU(wantU ? cnt : 0), pV(wantV ? cnt : 0);
    std::vector<int> ld_(cnt);
    for (int i = 0; i < cnt; ++i) {
      const int b = b0 + i;
      pA[i] = dA + oA[b];
      ld_[i] = m[b];
      pS[i] = dS + oS[b];
      if (wantU) pU[i] = dU + oU[b];
      if (wantV) pV[i] = dV + oV[b];
    }
    wcsvd_opts o;
    std::memset(&o, 0, sizeof(o));
    o.struct_size = sizeof(o);
    o.info = h_info ? dI : nullptr;
    if (opts) {
      o.force_path = opts->force_path;
      o.force_w = opts->force_w;
      o.wcycle_sweeps = opts->wcycle_sweeps;
      o.inner_sweeps = opts->inner_sweeps;
      o.pair_warps = opts->pair_warps;
      o.cluster_ctas = opts->cluster_ctas;
      o.f32_compute = opts->f32_compute;
    }
    rc = batched_impl<double>(cnt, m + b0, n + b0, pA.data(), ld_.data(), pS.data(), wantU ? pU.data() : nullptr,
                              wantV ? pV.data() : nullptr, tol, max_sweeps,
                              reinterpret_cast<wcsvd_stream_t>(s_cp[cs]), &o, tot);
    if (rc != WCSVD_OK) break;
    e = cudaEventRecord(ev_cp[st], s_cp[cs]);
    // D2H of the previous chunk now (a copy to pageable host memory returns only when it is done, so
    // it is issued after this chunk's kernels are queued), this chunk's after the loop / next round
    if (e == cudaSuccess && c >= 1) e = d2h(c - 1);
  }
  if (e == cudaSuccess && rc == WCSVD_OK) e = d2h(C - 1);
  // join into `stream`, free the staging there, and wait for the host copies (synchronous API)
  const cudaStream_t joins[4] = {s_cp[0], s_cp[1], s_in, s_out};
  for (int i = 0; i < 4; ++i) {
    cudaEventRecord(hp->ev_join[i], joins[i]);
    cudaStreamWaitEvent(stream, hp->ev_join[i], 0);
  }
  cudaFreeAsync(dbuf, stream);
  const cudaError_t es2 = cudaStreamSynchronize(stream);
  if (rc != WCSVD_OK) return rc;
  if (e != cudaSuccess || es2 != cudaSuccess) {
    if (std::getenv("WCSVD_DEBUG"))
      std::fprintf(stderr, "wcsvd_batched_host: %s / %s\n", cudaGetErrorString(e), cudaGetErrorString(es2));
    cudaGetLastError();
    return WCSVD_ECUDA;
  }
  return WCSVD_OK;
}


extern "C" {

const char* wcsvd_version(void) { return "wcsvd 0.1 sm_100a"; }

const char* wcsvd_status_string(int status) {
  if (status == WCSVD_OK) return kStatus[0];
  if (status == WCSVD_ENOTSUP) return kStatus[2];
  if (status == WCSVD_ECUDA) return kStatus[3];
  if (status == WCSVD_ENOMEM) return kStatus[4];
  if (status < 0 && status >= -12) return kStatus[1];
  return "unknown status";
}

int wcsvd_plan(int m, int n, int force_path, int force_w, wcsvd_plan_t* out) {
  if (m < 1) return -1;
  if (n < 1) return -2;
  if (!out) return -5;
  if (m > kMaxDim || n > kMaxDim) return WCSVD_ENOTSUP;
  return plan_one(m, n, force_path, force_w, out);
}

int wcsvd_round_robin(int np, int step, int* pairs) {
  if (np < 2 || (np & 1) || step < 0 || step >= np - 1 || !pairs) return -1;
  for (int k = 0; k < np / 2; ++k) {
    const int a = rr_content(2 * k, step, np), b = rr_content(2 * k + 1, step, np);
    pairs[2 * k] = std::min(a, b);
    pairs[2 * k + 1] = std::max(a, b);
  }
  return 0;
}

size_t wcsvd_workspace_size(int batch, const int* m, const int* n) {
  if (batch <= 0 || !m || !n) return 0;
  for (int b = 0; b < batch; ++b)
    if (m[b] < 1 || n[b] < 1 || m[b] > kMaxDim || n[b] > kMaxDim) return 0;
  CallPlan cp;
  if (make_call_plan(batch, m, n, 0, 0, 0, nullptr, &cp) != WCSVD_OK) return 0;
  return cp.bytes;
}

int wcsvd_etkf_analysis(int batch, const int* m, const int* n, const double* const* S, const double* const* U,
                        const double* const* V, const double* const* d, double* const* wbar, double* const* T,
                        wcsvd_stream_t stream_) {
  cudaStream_t stream = reinterpret_cast<cudaStream_t>(stream_);
  if (batch < 0) return -1;
  if (batch == 0) return WCSVD_OK;
  if (!m) return -2;
  if (!n) return -3;
  if (!S) return -4;
  if (!U) return -5;
  if (!V) return -6;
  if (!d) return -7;
  if (!wbar) return -8;
  if (!T) return -9;
  int kmax = 0;
  std::vector<DaDesc> h(batch);
  for (int b = 0; b < batch; ++b) {
    if (m[b] < 1) return -2;
    if (n[b] < 1) return -3;
    if (!S[b]) return -4;
    if (!U[b]) return -5;
    if (!V[b]) return -6;
    if (!d[b]) return -7;
    if (!wbar[b]) return -8;
    if (!T[b]) return -9;
    if (m[b] > kMaxDim || n[b] > kMaxDim) return WCSVD_ENOTSUP;
    h[b] = DaDesc{S[b], U[b], V[b], d[b], wbar[b], T[b], m[b], n[b]};
    kmax = std::max(kmax, std::min(m[b], n[b]));
  }
  void* ws = nullptr;
  if (lib_malloc(&ws, sizeof(DaDesc) * (size_t)batch, stream) != cudaSuccess) {
    cudaGetLastError();
    return WCSVD_ENOMEM;
  }
  cudaError_t e = cudaMemcpyAsync(ws, h.data(), sizeof(DaDesc) * (size_t)batch, cudaMemcpyHostToDevice, stream);
  if (e == cudaSuccess) e = launch_etkf(static_cast<const DaDesc*>(ws), batch, kmax, stream);
  cudaFreeAsync(ws, stream);
  if (e != cudaSuccess) {
    cudaGetLastError();
    return WCSVD_ECUDA;
  }
  return WCSVD_OK;
}

int wcsvd_trim_workspace(void) {
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess) {
    cudaGetLastError();
    return WCSVD_ECUDA;
  }
  std::lock_guard<std::mutex> lk(g_pool_mu);
  if (dev >= 0 && dev < 64 && g_pools[dev] && cudaMemPoolTrimTo(g_pools[dev], 0) != cudaSuccess) {
    cudaGetLastError();
    return WCSVD_ECUDA;
  }
  return WCSVD_OK;
}

int wcsvd_batched_ex(int batch, const int* m, const int* n, const double* const* A, const int* lda,
                     double* const* S, double* const* U, double* const* V, double tol,
                     int max_sweeps, wcsvd_stream_t stream, const wcsvd_opts* opts) {
  return batched_impl<double>(batch, m, n, A, lda, S, U, V, tol, max_sweeps, stream, opts);
}

int wcsvd_batched(int batch, const int* m, const int* n, const double* const* A, const int* lda,
                  double* const* S, double* const* U, double* const* V, double tol, int max_sweeps,
                  wcsvd_stream_t stream) {
  return batched_impl<double>(batch, m, n, A, lda, S, U, V, tol, max_sweeps, stream, nullptr);
}

int wcsvd_batched_f32_ex(int batch, const int* m, const int* n, const float* const* A, const int* lda,
                         float* const* S, float* const* U, float* const* V, float tol, int max_sweeps,
                         wcsvd_stream_t stream, const wcsvd_opts* opts) {
  return batched_impl<float>(batch, m, n, A, lda, S, U, V, (double)tol, max_sweeps, stream, opts);
}

int wcsvd_batched_f32(int batch, const int* m, const int* n, const float* const* A, const int* lda,
                      float* const* S, float* const* U, float* const* V, float tol, int max_sweeps,
                      wcsvd_stream_t stream) {
  return batched_impl<float>(batch, m, n, A, lda, S, U, V, (double)tol, max_sweeps, stream, nullptr);
}

int wcsvd_batched_host(int batch, const int* m, const int* n, const double* const* A, const int* lda,
                       double* const* S, double* const* U, double* const* V, double tol, int max_sweeps,
                       wcsvd_stream_t stream, const wcsvd_opts* opts) {
  return batched_host_impl(batch, m, n, A, lda, S, U, V, tol, max_sweeps, stream, opts);
}

}  // extern "C"
