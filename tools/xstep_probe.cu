// Development probe: cycles per X step of the two-phase Level-0 kernel (l0_tp.cu x_step) for one
// CTA alone on an SM, on synthetic data, and of its parts. Prints one JSON object.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -I include
//        -I paper_conf_sc_xiaopxsmmlzt22_b200/csrc -o xstep_probe tools/xstep_probe.cu
#include "../paper_conf_sc_xiaopxsmmlzt22_b200/csrc/l0_tp.cu"

#include <cstdio>

using namespace wcsvd;

// MODE 0: full x_step; 1: skip the serial section (rotations stay from the init); 2: serial
// section only (phase 1 and rotate skipped).
template <int MODE>
__global__ void __launch_bounds__(128, 1) xprobe(long long* out, int sweeps) {
  constexpr int NP = 64, G = 8, R = 4, NL = NP / G, LP = NL / 2;
  extern __shared__ __align__(16) unsigned char smem[];
  const int RW4 = 16, PS = 33;
  double* part = reinterpret_cast<double*>(smem);
  double* nrm = part + 3 * RW4 * PS;
  double2* rot = reinterpret_cast<double2*>(nrm + 2 * NP);
  int* flag = reinterpret_cast<int*>(rot + (NP - 1) * G * (LP + 1));
  for (int i = threadIdx.x; i < 3 * RW4 * PS; i += blockDim.x) part[i] = 0.0;
  for (int i = threadIdx.x; i < (NP - 1) * G * (LP + 1); i += blockDim.x) rot[i] = make_double2(0.8, 0.6);
  for (int i = threadIdx.x; i < 2 * NP; i += blockDim.x) nrm[i] = 1.0 + i;
  __syncthreads();
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  TPCtx<double> cx;
  cx.part = part;
  cx.nrm = nrm;
  cx.rot = rot;
  cx.RW4 = RW4;
  cx.PS = PS;
  cx.lane = lane;
  cx.warp = MODE == 1 ? 99 : warp;
  cx.g = tid % G;
  cx.rt = tid / G;
  cx.isW = MODE != 2;
  cx.dtop = rr_dest(2 * lane, NP);
  cx.dbot = rr_dest(2 * lane + 1, NP);
  cx.tol2 = 1e-30;
  cx.par = 0;
  cx.nwarp = 4;
  cx.rot_flag = flag;
#ifdef WCSVD_PHASE_PROFILE
  cx.acc[0] = cx.acc[1] = cx.acc[2] = 0;
#endif
  double a[R][NL], b[R][NL];
  for (int r = 0; r < R; ++r)
    for (int l = 0; l < NL; ++l) a[r][l] = 0.01 * ((tid * 7 + r * 13 + l * 5) % 17) - 0.08;
  long long t0 = clock64();
  for (int s = 0; s < sweeps; ++s) x_sweep<double, NP, G, R>(cx, a, b), x_sweep<double, NP, G, R>(cx, b, a);
  long long t1 = clock64();
  double acc = 0;
  for (int r = 0; r < R; ++r)
    for (int l = 0; l < NL; ++l) acc += a[r][l];
  if (acc == 1234.5) out[3] = 1;
  if (tid == 0) out[0] = t1 - t0;
}

template <int MODE>
void run(const char* name, long long* d, bool last = false) {
  const int sweeps = 20;
  const size_t smem = 8 * (3 * 16 * 33 + 128) + 16 * 63 * 8 * 5 + 64;
  cudaFuncSetAttribute(xprobe<MODE>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  xprobe<MODE><<<1, 128, smem>>>(d, sweeps);
  xprobe<MODE><<<1, 128, smem>>>(d, sweeps);
  cudaError_t e = cudaDeviceSynchronize();
  long long h[4];
  cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
  printf("  \"%s\": %.1f%s\n", e == cudaSuccess ? name : cudaGetErrorString(e), (double)h[0] / (sweeps * 2 * 63), last ? "" : ",");
}

int main() {
  long long* d;
  cudaMalloc(&d, 64);
  printf("{\n");
  run<0>("x_step_full", d);
  run<1>("x_step_no_serial", d);
  run<2>("x_step_serial_only", d, true);
  printf("}\n");
  return 0;
}
