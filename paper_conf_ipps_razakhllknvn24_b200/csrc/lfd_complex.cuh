// lfd_complex.cuh -- complex128 helpers for the sm_100a kernels (double2 = (re, im)).
#pragma once
#include <cuda_runtime.h>

namespace lfd {

__device__ __forceinline__ double2 cz() { return make_double2(0.0, 0.0); }

// a * b
__device__ __forceinline__ double2 cmul(double2 a, double2 b) {
  return make_double2(fma(a.x, b.x, -a.y * b.y), fma(a.x, b.y, a.y * b.x));
}
// a * b + c
__device__ __forceinline__ double2 cfma(double2 a, double2 b, double2 c) {
  return make_double2(fma(a.x, b.x, fma(-a.y, b.y, c.x)), fma(a.x, b.y, fma(a.y, b.x, c.y)));
}
// a * x + b * y  (one row of a 2x2 pair block)
__device__ __forceinline__ double2 crow(double2 a, double2 x, double2 b, double2 y) {
  return cfma(a, x, cmul(b, y));
}
// conj(a) * b
__device__ __forceinline__ double2 cconjmul(double2 a, double2 b) {
  return make_double2(fma(a.x, b.x, a.y * b.y), fma(a.x, b.y, -a.y * b.x));
}

}  // namespace lfd
