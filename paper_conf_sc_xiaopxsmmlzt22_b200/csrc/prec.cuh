// prec.cuh -- arithmetic type traits of the Level-0 kernels: double (wcsvd_batched) or float
// (wcsvd_batched_f32).
#pragma once

#include <cuda_runtime.h>

namespace wcsvd {

// Arithmetic type traits: the kernel runs in double (wcsvd_batched) or float (wcsvd_batched_f32).
template <typename T>
struct Prec;
template <>
struct Prec<double> {
  using V2 = double2;
  static constexpr double eps = 1.1102230246251565404e-16;  // 2^-53
  __device__ static double2 mk(double a, double b) { return make_double2(a, b); }
  __device__ static double qnan() { return __longlong_as_double(0x7ff8000000000000ULL); }
};
template <>
struct Prec<float> {
  using V2 = float2;
  static constexpr float eps = 5.9604644775390625e-08f;  // 2^-24
  __device__ static float2 mk(float a, float b) { return make_float2(a, b); }
  __device__ static float qnan() { return __int_as_float(0x7fc00000); }
};

}  // namespace wcsvd
