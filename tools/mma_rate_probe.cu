// Probe: tcgen05.mma (kind::f16, cta_group::1, M = 128, K = 16, SS operands)
// issue rate vs N and vs the number of independent accumulators the chain
// rotates through (1 = every MMA accumulates into the same TMEM columns).
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/mp tools/mma_rate_probe.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

constexpr int NMMA = 8192;

__device__ __forceinline__ uint64_t desc(uint32_t saddr) {
  uint64_t d = 0;
  d |= (uint64_t)((saddr >> 4) & 0x3FFF);
  d |= (uint64_t)1 << 16;
  d |= (uint64_t)(1024 >> 4) << 32;
  d |= (uint64_t)1 << 46;
  d |= (uint64_t)2 << 61;
  return d;
}

__global__ void __launch_bounds__(128, 1) probe(int N, int nacc, int M, int issuers, int tf32, long long *cyc, int variant, int nst) {
  extern __shared__ __align__(1024) uint8_t sm[];
  uint8_t *s = (uint8_t *)(((uintptr_t)sm + 1023) & ~(uintptr_t)1023);
  __shared__ uint32_t tptr;
  __shared__ __align__(8) uint64_t bars[4];
  const int warp = threadIdx.x / 32;
  for (int i = threadIdx.x; i < 64 * 1024 / 4; i += blockDim.x) ((uint32_t *)s)[i] = 0x3f803f80u;
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(
        (uint32_t)__cvta_generic_to_shared(&tptr)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  if (threadIdx.x < 4)
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"((uint32_t)__cvta_generic_to_shared(&bars[threadIdx.x])));
  asm volatile("fence.proxy.async.shared::cta;\nfence.mbarrier_init.release.cluster;" ::: "memory");
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  const uint32_t tm = tptr;
  const uint32_t sa = (uint32_t)__cvta_generic_to_shared(s), sb = sa + 16384;
  const uint32_t fmt = tf32 ? 2u : 1u;
  const uint32_t idesc = (1u << 4) | (fmt << 7) | (fmt << 10) | ((uint32_t)(N >> 3) << 17) |
                         ((uint32_t)(M >> 4) << 24);
  __syncthreads();
  long long t0 = clock64();
  const int lane = threadIdx.x & 31;
  if (issuers == 0 && warp == 0) {
    // unrolled: 8 MMAs per iteration, descriptor offsets are immediates, one elected lane
    const uint64_t ad = desc(sa), bd = desc(sb);
    const uint32_t d = tm;
    bool leader;
    {
      uint32_t pred = 0;
      asm volatile("{\n.reg .pred P;\nelect.sync _|P, 0xffffffff;\nselp.u32 %0, 1, 0, P;\n}" : "=r"(pred));
      leader = pred != 0;
    }
    const uint32_t done = (uint32_t)__cvta_generic_to_shared(&bars[3]);
    const uint32_t cbar = (uint32_t)__cvta_generic_to_shared(&bars[2]);
    if (variant >= 2 && leader) asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(done) : "memory");
    __syncwarp();
    uint32_t stage = 0;
    for (int i = 0; i < NMMA; i += 4) {
      if (variant >= 2) {   // wait on a completed barrier (phase 0 done), as the FULL wait
        asm volatile("{\n.reg .pred P;\nW%=: mbarrier.try_wait.parity.shared::cta.b64 P, [%0], 0;\n@!P bra W%=;\n}" ::"r"(done) : "memory");
        asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
      }
      const uint64_t soff = variant >= 3 ? (uint64_t)(stage * 1024) : 0;   // runtime stage offset (16 B units)
      if (leader) {
#pragma unroll
        for (int j = 0; j < 4; ++j)
          asm volatile(
              "{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\n"
              "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n}\n" ::"r"(d),
              "l"(ad + soff + 2 * j), "l"(bd + soff + 2 * j), "r"(idesc), "r"(i + j));
        if (variant >= 1)
          asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(cbar));
      }
      __syncwarp();
      if (++stage == (uint32_t)nst) stage = 0;
    }
    if (leader) {
      asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(
          (uint32_t)__cvta_generic_to_shared(&bars[0])));
      asm volatile("{\n.reg .pred P;\nW: mbarrier.try_wait.parity.shared::cta.b64 P, [%0], 0;\n@!P bra W;\n}" ::"r"(
          (uint32_t)__cvta_generic_to_shared(&bars[0])));
    }
    __syncwarp();
  }
  if (lane == 0 && warp < issuers) {
    const uint64_t ad = desc(sa), bd = desc(sb);
    const int per = NMMA / issuers;
    for (int i = 0; i < per; ++i) {
      const uint32_t d = tm + (uint32_t)((((i % nacc) * issuers) + warp) * N);
      const uint32_t k = (uint32_t)(i & 3) * 2;   // walk K inside the 128 B row
      if (tf32)
        asm volatile(
            "{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\n"
            "tcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n}\n" ::"r"(d),
            "l"(ad + k), "l"(bd + k), "r"(idesc), "r"(i >= nacc ? 1 : 0));
      else
        asm volatile(
            "{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\n"
            "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n}\n" ::"r"(d),
            "l"(ad + k), "l"(bd + k), "r"(idesc), "r"(i >= nacc ? 1 : 0));
    }
    {
      uint64_t &bar = bars[warp];
      asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(
          (uint32_t)__cvta_generic_to_shared(&bar)));
      asm volatile("{\n.reg .pred P;\nW: mbarrier.try_wait.parity.shared::cta.b64 P, [%0], 0;\n@!P bra W;\n}" ::"r"(
          (uint32_t)__cvta_generic_to_shared(&bar)));
    }
  }
  __syncthreads();
  if (threadIdx.x == 0) cyc[blockIdx.x] = clock64() - t0;
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(tm));
}

int main() {
  long long *cyc, h[148];
  cudaMalloc(&cyc, sizeof(h));
  cudaFuncSetAttribute(probe, cudaFuncAttributeMaxDynamicSharedMemorySize, 80 * 1024);
  struct Cfg { int N, nacc, M, iss, tf32, var; };
  const Cfg cfgs[] = {{64, 1, 128, 0, 0, 0}, {64, 1, 128, 0, 0, 1}, {64, 1, 128, 0, 0, 2}, {64, 1, 128, 0, 0, 3},
                      {128, 1, 128, 0, 0, 3}, {256, 1, 128, 0, 0, 3}, {64, 1, 64, 0, 0, 0}, {32, 1, 64, 0, 0, 0}};
  for (const Cfg &c : cfgs) {
    {
      const int N = c.N, nacc = c.nacc;
      probe<<<148, 128, 80 * 1024>>>(N, nacc, c.M, c.iss, c.tf32, cyc, c.var, 3);
      cudaError_t e = cudaDeviceSynchronize();
      if (e != cudaSuccess) { printf("err %s\n", cudaGetErrorString(e)); return 1; }
      cudaMemcpy(h, cyc, sizeof(h), cudaMemcpyDeviceToHost);
      double avg = 0;
      for (int i = 0; i < 148; ++i) avg += h[i];
      avg /= 148;
      const double ideal = (double)c.M * N * (c.tf32 ? 8 : 16) / (c.tf32 ? 2048 : 4096);
      printf("var %d M %3d N %3d nacc %d issuers %d(0=unrolled) %s: %.1f cyc/MMA (ideal %.0f) -> %.0f%% of peak\n", c.var, c.M, N,
             nacc, c.iss, c.tf32 ? "tf32" : "bf16", avg / NMMA, ideal, 100 * ideal / (avg / NMMA));
      fflush(stdout);
    }
  }
  return 0;
}
