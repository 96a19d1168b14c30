// Development probe: cycles per inner-EVD step of the Level-1 kernel (l1_gram.cu evd_step, 2w = 32),
// for E EVD warps per SM, with or without co-resident warps that keep the FP64 pipe busy with DMMA.
// Every EVD starts from a fresh dense symmetric B (all 31 steps rotate). Prints one JSON object.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -I include
//        -I paper_conf_sc_xiaopxsmmlzt22_b200/csrc -o evd_probe tools/evd_probe.cu
#include <cstdio>

#include "../paper_conf_sc_xiaopxsmmlzt22_b200/csrc/l1_gram.cu"

using namespace wcsvd;
constexpr int W2 = 32;

__global__ void evd_probe(int n_evd_warps, int hog, int reps, long long* out, double* sink) {
  extern __shared__ __align__(16) unsigned char sm[];
  __shared__ volatile int done;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (threadIdx.x == 0) done = 0;
  __syncthreads();
  if (warp < n_evd_warps) {
    double* B0 = reinterpret_cast<double*>(sm) + warp * (2 * W2 * W2 + W2);
    double* B1 = B0 + W2 * W2;
    double2* cs = reinterpret_cast<double2*>(B1 + W2 * W2);
    EvdMap<W2> em;
    em.init(lane);
    double ja[W2], jb[W2];
    long long cyc = 0;
    double acc = 0.0;
    for (int rep = 0; rep < reps; ++rep) {
      for (int e = lane; e < W2 * W2; e += 32) {
        const int a = e / W2, b = e % W2;
        if (a <= b) B0[evd_phys<W2>(a, b)] = (a == b) ? 1.0 + 0.03 * a : 0.01 * ((a * 7 + b * 13 + rep) % 17 - 8);
      }
#pragma unroll
      for (int s = 0; s < W2; ++s) ja[s] = (lane == s) ? 1.0 : 0.0;
      __syncwarp();
      const long long t0 = clock64();
      bool any = evd_step<W2>(B0, B1, cs, em, lane, 1e-30, ja, jb);
      __syncwarp();
      for (int r = 1; r < W2 - 1; r += 2) {
        any |= evd_step<W2>(B1, B0, cs, em, lane, 1e-30, jb, ja);
        __syncwarp();
        any |= evd_step<W2>(B0, B1, cs, em, lane, 1e-30, ja, jb);
        __syncwarp();
      }
      cyc += clock64() - t0;
#pragma unroll
      for (int s = 0; s < W2; ++s) acc += jb[s];
      acc += any ? 1.0 : 0.0;
    }
    if (lane == 0) out[blockIdx.x * 32 + warp] = cyc;
    sink[blockIdx.x * blockDim.x + threadIdx.x] = acc;
    __syncthreads();  // all EVD warps done
    if (threadIdx.x == 0) done = 1;
  } else {
    __syncthreads();
    if (!hog) return;
    double c[4][2];
#pragma unroll
    for (int i = 0; i < 4; ++i) c[i][0] = c[i][1] = i;
    const double a = 0.5 + lane, b = 0.25;
    while (!done) {
#pragma unroll
      for (int i = 0; i < 4; ++i) dmma884(c[i], a, b);
    }
    sink[blockIdx.x * blockDim.x + threadIdx.x] = c[0][0] + c[1][1] + c[2][0] + c[3][1];
  }
}

int main() {
  long long* d;
  double* sink;
  cudaMalloc(&d, 148 * 32 * sizeof(long long));
  cudaMalloc(&sink, 148 * 1024 * sizeof(double));
  const int reps = 20;
  const size_t smem = 8 * (2 * W2 * W2 + W2) * sizeof(double);
  cudaFuncSetAttribute(evd_probe, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  printf("{\n");
  const int cfg[][2] = {{1, 0}, {4, 0}, {4, 4}, {8, 0}, {2, 2}, {6, 2}};  // <= 8 warps (255 regs)
  for (int i = 0; i < 6; ++i) {
    const int ne = cfg[i][0], nh = cfg[i][1];
    for (int warm = 0; warm < 2; ++warm) {
      evd_probe<<<148, 32 * (ne + nh), smem>>>(ne, nh > 0, reps, d, sink);
      cudaDeviceSynchronize();
    }
    long long h[148 * 32];
    cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
    double tot = 0;
    for (int b = 0; b < 148; ++b)
      for (int w = 0; w < ne; ++w) tot += h[b * 32 + w];
    const double per_step = tot / (148.0 * ne * reps * (W2 - 1));
    printf("  \"evd%d_hog%d\": {\"cycles_per_step\": %.1f}%s\n", ne, nh, per_step, i == 5 ? "" : ",");
  }
  printf("}\n");
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) fprintf(stderr, "%s\n", cudaGetErrorString(e));
  return 0;
}
