// lrn_math.cuh -- the LRN arithmetic shared by the stand-alone LRN/pool
// kernels and the conv epilogue that fuses LRN (all must compute identically):
// b_c = a_c / (k + alpha/n * sum_window a^2)^beta  (R3).
#pragma once
#include <stdint.h>

namespace pcnn {

// The LRN of N consecutive channels: out[j] = x[j] * (k + a_n *
// sum_{w<LS} sq[j+w])^(-beta), with sq[t] = the square of channel j0 + t -
// LS/2 (zero outside the tensor), computed by every caller as __fmul_rn(x, x)
// so no caller's compiler can contract it into the window sum.  Every LRN path (the stand-alone kernels and
// the conv epilogue) calls this, so they agree bit for bit.
//   * size 5: the window is summed as ((sq0 + sq1) + (sq2 + sq3)) + sq4, so
//     neighbouring channels share the pair sums and the dependency chain is
//     3 adds deep instead of 5;
//   * s^-beta = 2^(-beta log2 s) with the MUFU approximations (relative error
//     ~2^-22, far inside the FP32 tolerance of 1e-4).
template <bool BF16, int LS, int N>
__device__ __forceinline__ void lrn_normalise(const float *sq, const float *x, float k,
                                              float a_n, float beta, float *out) {
  float scale[N];
#pragma unroll
  for (int j = 0; j < N; ++j) {
    float acc;
    if constexpr (LS == 5) {
      acc = ((sq[j] + sq[j + 1]) + (sq[j + 2] + sq[j + 3])) + sq[j + 4];
    } else {
      acc = 0.f;
#pragma unroll
      for (int w = 0; w < LS; ++w) acc += sq[j + w];
    }
    scale[j] = k + a_n * acc;
  }
#pragma unroll
  for (int j = 0; j < N; ++j) {
    float l, r;
    asm("lg2.approx.ftz.f32 %0, %1;" : "=f"(l) : "f"(scale[j]));
    asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(-beta * l));
    out[j] = x[j] * r;
  }
}

// Exact q = v / d, r = v % d for 0 <= v < 2^22 and d <= 2^10 via a float
// reciprocal inv = 1/d (precomputed): (v + 0.5) * inv never rounds across an
// integer at these magnitudes.
__device__ __forceinline__ void fdivmod(int v, int d, float inv, int &q, int &r) {
  q = __float2int_rz(((float)v + 0.5f) * inv);
  r = v - q * d;
}

}  // namespace pcnn
