// budget.cuh -- per-layer SM / CTA budget on the device side.
//
// The paper's run-time kernel scheduler gives each layer optSM SMs and puts
// optTLP CTAs on each before moving to the next SM (Priority-SM, P:213,
// Fig. 7).  On B200 the hardware CTA scheduler is breadth-first, so:
//   * tcgen05 kernels are 1 CTA/SM by construction (smem + TMEM); a grid cap
//     of n CTAs running a persistent tile loop occupies exactly n SMs.
//   * SIMT kernels launch a full wave; a CTA is admitted only if its %smid is
//     below n and fewer than tlp CTAs were admitted on that SM, and admitted
//     CTAs pull tiles from an atomic counter until the layer is done.
// Tiles never split the K reduction, so every budget gives bitwise identical
// results (R11).
#pragma once
#include "pcnn_internal.h"

namespace pcnn {

__device__ __forceinline__ unsigned smid_u32() {
  unsigned r;
  asm volatile("mov.u32 %0, %%smid;" : "=r"(r));
  return r;
}

__device__ __forceinline__ void census_mark(const Budget &b) {
  if (b.census) {
    unsigned id = smid_u32();
    if (id < (unsigned)kMaxSMs) atomicOr(&b.census[id >> 5], 1u << (id & 31));
  }
}

// Block-uniform admission; must be called by all threads of the CTA.
__device__ __forceinline__ bool budget_admit(const Budget &b, int *sh_flag) {
  if (!b.gated) {
    if (threadIdx.x == 0) census_mark(b);
    return true;
  }
  if (threadIdx.x == 0) {
    unsigned id = smid_u32();
    int ok = 0;
    if ((int)id < b.n_sms) {
      unsigned long long slot = atomicAdd(&b.ctr[1 + id], 1ULL);
      ok = slot < (unsigned long long)b.tlp;
    }
    if (ok) census_mark(b);
    *sh_flag = ok;
  }
  __syncthreads();
  return *sh_flag != 0;
}

// Tile loop for SIMT kernels.  body(t) is called by all threads of the CTA.
template <typename F>
__device__ __forceinline__ void for_each_tile(const Budget &b, long long tiles,
                                              F body) {
  __shared__ int sh_flag;
  __shared__ long long sh_tile;
  if (!budget_admit(b, &sh_flag)) return;
  if (!b.gated) {
    for (long long t = blockIdx.x; t < tiles; t += gridDim.x) body(t);
    return;
  }
  for (;;) {
    __syncthreads();
    if (threadIdx.x == 0) sh_tile = (long long)atomicAdd(&b.ctr[0], 1ULL);
    __syncthreads();
    const long long t = sh_tile;
    if (t >= tiles) break;
    body(t);
  }
}

}  // namespace pcnn
