// lrn_math.cuh -- the LRN scale shared by the stand-alone LRN/pool kernel and
// the conv epilogue that fuses LRN (both must compute identically).
#pragma once

namespace pcnn {

// x * (k + alpha/n * sum_window x^2)^(-beta)   (R3)
// s^(-beta) = 2^(-beta * log2 s) with the MUFU approximations (relative error
// ~2^-22, far inside the FP32 tolerance of 1e-4).
__device__ __forceinline__ float lrn_scale_pow(float scale, float beta) {
  float l, r;
  asm("lg2.approx.ftz.f32 %0, %1;" : "=f"(l) : "f"(scale));
  asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(-beta * l));
  return r;
}

// Exact q = v / d, r = v % d for 0 <= v < 2^22 and d <= 2^10 via a float
// reciprocal inv = 1/d (precomputed): (v + 0.5) * inv never rounds across an
// integer at these magnitudes.
__device__ __forceinline__ void fdivmod(int v, int d, float inv, int &q, int &r) {
  q = __float2int_rz(((float)v + 0.5f) * inv);
  r = v - q * d;
}

}  // namespace pcnn
