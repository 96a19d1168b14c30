// Latency microbenchmark (development probe): dependent-chain latency in cycles of the FP64 /
// FP32 operations on the Jacobi rotation's critical path, for one warp alone on an SM and with a
// DMMA-saturating warp co-resident on the same SMSP. Prints one JSON object.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o lat tools/lat_fp64.cu
#include <cstdio>
#include <cuda_runtime.h>

constexpr int ITERS = 256;

enum Op { DFMA, DADD, DMUL, DSQRT, DRSQRT, DRCP, DDIV, FFMA, FSQRT, FRSQRT, SHFL64, LDS64, RSQ64H, DFMA8, NOPS };
static const char* names[NOPS] = {"dfma", "dadd", "dmul", "dsqrt", "drsqrt", "drcp", "ddiv", "ffma",
                                  "fsqrt_rn", "frsqrt", "shfl64", "lds64", "rsq64h_approx", "dfma_ilp8_per_instr"};

__device__ __forceinline__ double rsq64h(double x) {
  double r;
  asm volatile("rsqrt.approx.ftz.f64 %0, %1;" : "=d"(r) : "d"(x));
  return r;
}

template <int OP>
__device__ __forceinline__ long long chain(double& v, float& f, double* sm) {
  double w[8];
#pragma unroll
  for (int j = 0; j < 8; ++j) w[j] = v + j;
  long long t0 = clock64();
#pragma unroll 16
  for (int i = 0; i < ITERS; ++i) {
    if (OP == DFMA) v = fma(v, 0.9999999, 1e-9);
    if (OP == DADD) v = v + 1e-9;
    if (OP == DMUL) v = v * 1.0000001;
    if (OP == DSQRT) v = sqrt(v) + 0.5;
    if (OP == DRSQRT) v = rsqrt(v) + 0.5;
    if (OP == DRCP) v = 1.0 / v + 0.5;
    if (OP == DDIV) v = 1.5 / v;
    if (OP == FFMA) f = fmaf(f, 0.9999f, 1e-6f);
    if (OP == FSQRT) f = __fsqrt_rn(f) + 0.5f;
    if (OP == FRSQRT) f = rsqrtf(f) + 0.5f;
    if (OP == SHFL64) v = __shfl_xor_sync(0xffffffffu, v, 1);
    if (OP == LDS64) v = sm[(int)v & 7];
    if (OP == RSQ64H) v = rsq64h(v) + 0.5;
    if (OP == DFMA8) {
#pragma unroll
      for (int j = 0; j < 8; ++j) w[j] = fma(w[j], 0.9999999, 1e-9);
    }
  }
  if (OP == DFMA8) {
#pragma unroll
    for (int j = 0; j < 8; ++j) v += w[j];
  }
  long long t1 = clock64();
  return t1 - t0;
}

template <int OP>
__global__ void lat_kernel(long long* out, double x, int hog_dmma) {
  __shared__ double sm[8];
  __shared__ volatile int done;
  if (threadIdx.x < 8) sm[threadIdx.x] = threadIdx.x & 7;
  if (threadIdx.x == 0) done = 0;
  __syncthreads();
  const int warp = threadIdx.x >> 5;
  if (warp == 0) {
    double v = x + 1.0;
    float f = (float)x + 1.0f;
    if (OP == LDS64) v = 1.0;
    long long c = chain<OP>(v, f, sm);
    c = chain<OP>(v, f, sm);  // second pass: warm instruction cache
    if (threadIdx.x == 0) out[0] = c;
    if (v == 12345.0 || f == 12345.0f) out[1] = 1;
    __syncwarp();
    if (threadIdx.x == 0) done = 1;
  } else if (hog_dmma) {
    // warp 4 shares SMSP 0 with warp 0: keep the FP64 pipe busy with independent DMMAs.
    if (warp != 4) return;
    double c[4][2];
#pragma unroll
    for (int i = 0; i < 4; ++i) c[i][0] = c[i][1] = i;
    const double a = x, b = x * 0.5;
    long long hog_t0 = clock64(), n = 0;
    while (!done) {
      ++n;
#pragma unroll
      for (int i = 0; i < 4; ++i)
        asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};"
                     : "+d"(c[i][0]), "+d"(c[i][1]) : "d"(a), "d"(b));
    }
    if (c[0][0] + c[1][1] + c[2][0] + c[3][1] == 12345.0) out[1] = 2;
    if ((threadIdx.x & 31) == 0) { out[2] = n * 4; out[3] = clock64() - hog_t0; }
  }
}

template <int OP>
double run(long long* d, int hog) {
  lat_kernel<OP><<<1, hog ? 160 : 32>>>(d, 0.37, hog);
  cudaDeviceSynchronize();
  long long h[4];
  cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
  if (hog) printf("  \"_hog_%d\": {\"dmma\": %lld, \"cycles\": %lld, \"cyc_per_dmma\": %.1f},\n", OP, h[2], h[3], (double)h[3] / (h[2] ? h[2] : 1));
  return (double)h[0] / ITERS / (OP == DFMA8 ? 8 : 1);
}

template <int OP>
void report(long long* d, bool last) {
  const double a = run<OP>(d, 0), b = run<OP>(d, 1);
  printf("  \"%s\": {\"alone\": %.1f, \"with_dmma_warp\": %.1f}%s\n", names[OP], a, b, last ? "" : ",");
}

int main() {
  long long* d;
  cudaMalloc(&d, 32);
  printf("{\n");
  report<DFMA>(d, false);
  report<DADD>(d, false);
  report<DMUL>(d, false);
  report<DSQRT>(d, false);
  report<DRSQRT>(d, false);
  report<DRCP>(d, false);
  report<DDIV>(d, false);
  report<RSQ64H>(d, false);
  report<FFMA>(d, false);
  report<FSQRT>(d, false);
  report<FRSQRT>(d, false);
  report<SHFL64>(d, false);
  report<LDS64>(d, false);
  report<DFMA8>(d, true);
  printf("}\n");
  return 0;
}
