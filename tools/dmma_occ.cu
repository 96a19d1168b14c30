// Microbenchmark: DMMA.8x8x4 throughput vs resident warps per SM and independent chains per warp.
#include <cstdio>
template <int ILP>
__global__ void dmma_loop(double* out, int iters) {
  double c[ILP][2];
  double a = 1.0 + threadIdx.x * 1e-9, b = 0.5;
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
template <int ILP> void run(int warps_per_sm, double* out) {
  int blocks = 148, threads = 32 * warps_per_sm, iters = 4096;
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  dmma_loop<ILP><<<blocks, threads>>>(out, iters);
  cudaEventRecord(e0);
  dmma_loop<ILP><<<blocks, threads>>>(out, iters);
  cudaEventRecord(e1); cudaEventSynchronize(e1);
  float ms; cudaEventElapsedTime(&ms, e0, e1);
  double flops = 2.0 * 256 * ILP * (double)iters * blocks * warps_per_sm;
  printf("warps/SM=%2d ILP=%d  %.2f TF/s\n", warps_per_sm, ILP, flops / (ms * 1e-3) / 1e12);
}
int main() {
  double* out; cudaMalloc(&out, 1 << 20);
  for (int w : {4, 8, 16, 32}) { run<1>(w, out); run<2>(w, out); run<4>(w, out); run<8>(w, out); }
  return 0;
}
