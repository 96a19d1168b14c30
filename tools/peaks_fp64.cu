// Step-0 microbenchmark: measure the FP64 roofline denominators on the
// B200 this run uses. MEASURED_PEAKS.json carries only HBM and bf16 numbers, and the method's hot
// path is fp64 (DFMA + DMMA.8x8x4; tcgen05 has no f64 kind). Prints one JSON object.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o peaks_fp64 tools/peaks_fp64.cu
#include <cstdio>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("{\"error\":\"%s\"}\n", cudaGetErrorString(e)); return 1; } } while (0)

template <int ILP>
__global__ void dfma_loop(double* out, int iters, double x) {
  double acc[ILP];
#pragma unroll
  for (int i = 0; i < ILP; ++i) acc[i] = x + i * 1e-3 + threadIdx.x * 1e-9;
  const double a = 0.999999, b = 1e-7;
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int i = 0; i < ILP; ++i) acc[i] = fma(acc[i], a, b);
  }
  double s = 0;
#pragma unroll
  for (int i = 0; i < ILP; ++i) s += acc[i];
  if (s == 1234.5) out[threadIdx.x] = s;
}

template <int ILP>
__global__ void dmma_loop(double* out, int iters, double x) {
  double c[ILP][2];
  double a = x + threadIdx.x * 1e-9, b = x * 0.5;
#pragma unroll
  for (int i = 0; i < ILP; ++i) { c[i][0] = i; c[i][1] = -i; }
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int i = 0; i < ILP; ++i)
      asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};"
                   : "+d"(c[i][0]), "+d"(c[i][1]) : "d"(a), "d"(b));
  }
  double s = 0;
#pragma unroll
  for (int i = 0; i < ILP; ++i) s += c[i][0] + c[i][1];
  if (s == 1234.5) out[threadIdx.x] = s;
}

__global__ void shfl_loop(double* out, int iters, double x) {
  double v[8];
#pragma unroll
  for (int i = 0; i < 8; ++i) v[i] = x + i + threadIdx.x;
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int i = 0; i < 8; ++i) v[i] = __shfl_xor_sync(0xffffffffu, v[i], 1 + (i & 15));
  }
  double s = 0;
#pragma unroll
  for (int i = 0; i < 8; ++i) s += v[i];
  if (s == 1234.5) out[threadIdx.x] = s;
}

__global__ void lds_loop(double* out, int iters) {
  __shared__ double sm[4096];
  for (int i = threadIdx.x; i < 4096; i += blockDim.x) sm[i] = i;
  __syncthreads();
  double s = 0;
  int idx = threadIdx.x;
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int i = 0; i < 8; ++i) s += sm[(idx + i * 256) & 4095];
    idx = (idx + 32) & 4095;
  }
  if (s == 1234.5) out[threadIdx.x] = s;
}

template <typename K>
float time_kernel(K kern, int blocks, int threads, int iters, double* out) {
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0); cudaEventCreate(&e1);
  kern<<<blocks, threads>>>(out, iters, 1.0);  // warm-up
  cudaEventRecord(e0);
  for (int r = 0; r < 5; ++r) kern<<<blocks, threads>>>(out, iters, 1.0);
  cudaEventRecord(e1);
  cudaEventSynchronize(e1);
  float ms; cudaEventElapsedTime(&ms, e0, e1);
  return ms / 5;
}

int main() {
  int dev = 0, sms = 0, clk = 0, l2 = 0, smem = 0;
  CK(cudaSetDevice(dev));
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, dev);
  cudaDeviceGetAttribute(&l2, cudaDevAttrL2CacheSize, dev);
  cudaDeviceGetAttribute(&smem, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
  double* out; CK(cudaMalloc(&out, 1 << 20));
  const int iters = 1 << 16;
  printf("{\"sms\": %d, \"clock_khz\": %d, \"l2_bytes\": %d, \"smem_optin\": %d", sms, clk, l2, smem);
  // DFMA: blocks = 4*sms, 256 threads, ILP 8
  {
    int blocks = sms * 4, threads = 256;
    float ms = time_kernel(dfma_loop<8>, blocks, threads, iters, out);
    double flops = 2.0 * 8 * iters * (double)blocks * threads;
    printf(", \"dfma_tflops\": %.3f", flops / (ms * 1e-3) / 1e12);
  }
  {
    int blocks = sms * 4, threads = 256;
    float ms = time_kernel(dmma_loop<4>, blocks, threads, iters / 4, out);
    double flops = 2.0 * 256 * 4 * (iters / 4) * (double)blocks * (threads / 32);
    printf(", \"dmma_tflops\": %.3f", flops / (ms * 1e-3) / 1e12);
  }
  {
    int blocks = sms * 4, threads = 256;
    float ms = time_kernel(dmma_loop<8>, blocks, threads, iters / 8, out);
    double flops = 2.0 * 256 * 8 * (iters / 8) * (double)blocks * (threads / 32);
    printf(", \"dmma_tflops_ilp8\": %.3f", flops / (ms * 1e-3) / 1e12);
  }
  {
    int blocks = sms * 4, threads = 256;
    float ms = time_kernel(shfl_loop, blocks, threads, iters / 4, out);
    double warp_shfl = 2.0 * 8 * (iters / 4) * (double)blocks * (threads / 32);  // 2 SHFL per double
    printf(", \"shfl32_warp_instr_per_clk_per_sm\": %.3f", warp_shfl / (ms * 1e-3) / (clk * 1e3) / sms);
  }
  {
    int blocks = sms * 4, threads = 256;
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
    lds_loop<<<blocks, threads>>>(out, iters / 4);
    cudaEventRecord(e0);
    lds_loop<<<blocks, threads>>>(out, iters / 4);
    cudaEventRecord(e1); cudaEventSynchronize(e1);
    float ms; cudaEventElapsedTime(&ms, e0, e1);
    double bytes = 8.0 * 8 * (iters / 4) * (double)blocks * threads;
    printf(", \"lds64_bytes_per_clk_per_sm\": %.2f", bytes / (ms * 1e-3) / (clk * 1e3) / sms);
  }
  CK(cudaGetLastError());
  printf("}\n");
  return 0;
}
