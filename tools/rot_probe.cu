// Development probe: cycles per round-robin step of the Level-0 rotate-and-move code path
// (l0_tp.cu rotate_move) in isolation, for one CTA of NT threads on one SM, with and without
// the barrier pair of the X phase. Prints one JSON object.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -I paper_conf_sc_xiaopxsmmlzt22_b200/csrc -o rot_probe tools/rot_probe.cu
#include <cstdio>
#include <cuda_runtime.h>

#include "prec.cuh"

using namespace wcsvd;

template <typename T, int NP, int G, int R, int SUB, bool SHUF>
__device__ __forceinline__ void rotate_move(const T (&x)[R][NP / G], T (&y)[R][NP / G],
                                            const double2* __restrict__ cs, int g) {
  constexpr int NL = NP / G;
  constexpr int LP = NL / 2;
  T top0[R], send_l[R], send_r[R];
#pragma unroll
  for (int j = 0; j < LP; ++j) {
    const double2 p = cs[(j / SUB) * (SUB + 1) + (j % SUB)];
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
    if (SHUF && G > 1) {
      from_left = __shfl_up_sync(0xffffffffu, send_r[r], 1);
      from_right = __shfl_down_sync(0xffffffffu, send_l[r], 1);
    }
    y[r][0] = gfirst ? top0[r] : from_left;
    y[r][2] = gfirst ? send_l[r] : top0[r];
    y[r][2 * (LP - 1) + 1] = glast ? send_r[r] : from_right;
  }
}

template <int NP, int G, int R, bool SHUF, int BARS>
__global__ void __launch_bounds__(128, 1) probe(long long* out, double seed, int steps) {
  constexpr int NL = NP / G, LP = NL / 2;
  __shared__ double2 cs[64 * G * (LP + 1)];
  for (int i = threadIdx.x; i < 64 * G * (LP + 1); i += blockDim.x) {
    const double t = 0.001 * (i % 7);
    cs[i] = make_double2(1.0 / sqrt(1 + t * t), t / sqrt(1 + t * t));
  }
  __syncthreads();
  const int g = threadIdx.x % G;
  double x[R][NL], y[R][NL];
#pragma unroll
  for (int r = 0; r < R; ++r)
#pragma unroll
    for (int l = 0; l < NL; ++l) x[r][l] = seed + r + 0.1 * l + threadIdx.x * 1e-3;
  long long t0 = clock64();
  for (int s = 0; s < steps; s += 2) {
    if (BARS) { __syncthreads(); if (BARS > 1) __syncthreads(); }
    rotate_move<double, NP, G, R, LP, SHUF>(x, y, cs + (s & 63) * G * (LP + 1) + g * (LP + 1), g);
    if (BARS) { __syncthreads(); if (BARS > 1) __syncthreads(); }
    rotate_move<double, NP, G, R, LP, SHUF>(y, x, cs + ((s + 1) & 63) * G * (LP + 1) + g * (LP + 1), g);
  }
  long long t1 = clock64();
  double acc = 0;
#pragma unroll
  for (int r = 0; r < R; ++r)
#pragma unroll
    for (int l = 0; l < NL; ++l) acc += x[r][l];
  if (acc == 1234.5) out[2] = 1;
  if (threadIdx.x == 0) out[0] = t1 - t0;
}

template <int NP, int G, int R, bool SHUF, int BARS>
void run(const char* name, long long* d, int nt, bool last = false) {
  const int steps = 4096;
  probe<NP, G, R, SHUF, BARS><<<1, nt>>>(d, 0.5, steps);
  probe<NP, G, R, SHUF, BARS><<<1, nt>>>(d, 0.5, steps);
  cudaDeviceSynchronize();
  long long h[3];
  cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
  printf("  \"%s_nt%d\": %.1f%s\n", name, nt, (double)h[0] / steps, last ? "" : ",");
}

int main() {
  long long* d;
  cudaMalloc(&d, 64);
  printf("{\n");
  run<64, 8, 4, true, 0>("g8r4_shfl", d, 32);
  run<64, 8, 4, true, 0>("g8r4_shfl", d, 128);
  run<64, 8, 4, false, 0>("g8r4_noshfl", d, 32);
  run<64, 8, 4, false, 0>("g8r4_noshfl", d, 128);
  run<64, 8, 4, true, 1>("g8r4_shfl_bar1", d, 128);
  run<64, 8, 4, true, 2>("g8r4_shfl_bar2", d, 128);
  run<64, 2, 1, true, 0>("g2r1_shfl", d, 32);
  run<64, 2, 1, true, 0>("g2r1_shfl", d, 128);
  run<64, 8, 8, true, 0>("g8r8_shfl", d, 32);
  run<64, 8, 8, true, 0>("g8r8_shfl", d, 64, true);
  printf("}\n");
  return 0;
}
