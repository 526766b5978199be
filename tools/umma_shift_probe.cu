// Probe: does a tcgen05 SW128 K-major A descriptor whose start address is
// advanced by s whole 128 B rows (s = 0..7, not a multiple of the 1024 B
// swizzle atom) read rows s..s+127 of the swizzled region?  Tried with the
// descriptor's base-offset field (bits 49-51) = 0 and = s & 7.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -o /tmp/usp tools/umma_shift_probe.cu
#include <cstdio>
#include <cstdint>
#include <cuda_bf16.h>

constexpr int ROWS = 136, N = 64, KMAX = 64;

// rows of RB bytes (128: SW128, 64: SW64), 8-row atoms every 8*RB bytes
__device__ uint64_t desc(uint32_t saddr, uint32_t base_off, int RB) {
  uint64_t d = 0;
  d |= (uint64_t)((saddr >> 4) & 0x3FFF);
  d |= (uint64_t)1 << 16;
  d |= (uint64_t)((8 * RB) >> 4) << 32;
  d |= (uint64_t)1 << 46;
  d |= (uint64_t)(base_off & 7) << 49;
  d |= (uint64_t)(RB == 128 ? 2 : 4) << 61;
  return d;
}
// swizzled byte offset of logical offset `a` inside a 1024-aligned region
__host__ __device__ uint32_t swz(uint32_t a, int RB) {
  const uint32_t m = RB == 128 ? 7 : 3;
  return a ^ (((a >> 7) & m) << 4);
}

__global__ void probe(const __nv_bfloat16 *A, const __nv_bfloat16 *B, float *D, int shift, int mode,
                      int RB) {
  const int K = RB / 2, CH = RB / 16;   // bf16 elements / 16 B chunks per row
  extern __shared__ __align__(1024) uint8_t sm[];
  uint8_t *s = (uint8_t *)(((uintptr_t)sm + 1023) & ~(uintptr_t)1023);
  uint8_t *sA = s, *sB = s + 17408;
  __shared__ uint32_t tptr;
  __shared__ uint64_t bar;
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  // SW128 fill: 16 B chunk j of row r lives at chunk j ^ (r & 7)
  for (int i = tid; i < ROWS * CH; i += blockDim.x) {
    int r = i / CH, j = i % CH;
    *(uint4 *)(sA + swz(r * RB + j * 16, RB)) = *(const uint4 *)(A + r * KMAX + j * 8);
  }
  for (int i = tid; i < N * CH; i += blockDim.x) {
    int r = i / CH, j = i % CH;
    *(uint4 *)(sB + swz(r * RB + j * 16, RB)) = *(const uint4 *)(B + r * KMAX + j * 8);
  }
  uint32_t sbar = (uint32_t)__cvta_generic_to_shared(&bar);
  if (tid == 0) asm volatile("mbarrier.init.shared.b64 [%0], 1;" ::"r"(sbar));
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 64;" ::"r"(
        (uint32_t)__cvta_generic_to_shared(&tptr)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;");
  const uint32_t tm = tptr;
  if (tid == 0) {
    const uint32_t aaddr = (uint32_t)__cvta_generic_to_shared(sA) + shift * RB;
    const uint32_t baddr = (uint32_t)__cvta_generic_to_shared(sB);
    const uint32_t idesc = (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(N >> 3) << 17) |
                           ((uint32_t)(128 >> 4) << 24);
    for (int k = 0; k < RB / 32; ++k) {
      uint64_t ad = desc(aaddr + 32 * k, mode ? (aaddr >> 7) : 0, RB);
      uint64_t bd = desc(baddr + 32 * k, 0, RB);
      asm volatile(
          "{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\n"
          "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n}\n" ::"r"(tm),
          "l"(ad), "l"(bd), "r"(idesc), "r"(k));
    }
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(sbar));
  }
  asm volatile(
      "{\n.reg .pred P1;\nW: mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], 0;\n@!P1 bra W;\n}\n" ::"r"(sbar));
  asm volatile("tcgen05.fence::after_thread_sync;");
  for (int c = 0; c < N; c += 8) {
    uint32_t v[8];
    asm volatile("tcgen05.ld.sync.aligned.32x32b.x8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                 : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]),
                   "=r"(v[6]), "=r"(v[7])
                 : "r"(tm + ((uint32_t)(warp * 32) << 16) + c));
    asm volatile("tcgen05.wait::ld.sync.aligned;");
    for (int i = 0; i < 8; ++i) D[(warp * 32 + lane) * N + c + i] = __uint_as_float(v[i]);
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 64;" ::"r"(tm));
}

int main() {
  static __nv_bfloat16 hA[ROWS * KMAX], hB[N * KMAX];
  static float fA[ROWS * KMAX], fB[N * KMAX], hD[128 * N];
  for (int i = 0; i < ROWS * KMAX; ++i) { fA[i] = (float)((i * 7 + 3) % 11 - 5); hA[i] = __float2bfloat16(fA[i]); }
  for (int i = 0; i < N * KMAX; ++i) { fB[i] = (float)((i * 5 + 1) % 7 - 3); hB[i] = __float2bfloat16(fB[i]); }
  __nv_bfloat16 *dA, *dB; float *dD;
  cudaMalloc(&dA, sizeof(hA)); cudaMalloc(&dB, sizeof(hB)); cudaMalloc(&dD, sizeof(hD));
  cudaMemcpy(dA, hA, sizeof(hA), cudaMemcpyHostToDevice);
  cudaMemcpy(dB, hB, sizeof(hB), cudaMemcpyHostToDevice);
  cudaFuncSetAttribute(probe, cudaFuncAttributeMaxDynamicSharedMemorySize, 40000);
  for (int RB = 128; RB >= 64; RB /= 2)
  for (int mode = 0; mode < 2; ++mode)
    for (int shift = 0; shift < 8; ++shift) {
      const int K = RB / 2;
      cudaMemset(dD, 0, sizeof(hD));
      probe<<<1, 128, 40000>>>(dA, dB, dD, shift, mode, RB);
      cudaError_t e = cudaDeviceSynchronize();
      if (e != cudaSuccess) { printf("mode %d shift %d: %s\n", mode, shift, cudaGetErrorString(e)); return 1; }
      cudaMemcpy(hD, dD, sizeof(hD), cudaMemcpyDeviceToHost);
      int bad = 0;
      for (int m = 0; m < 128; ++m)
        for (int n = 0; n < N; ++n) {
          float ref = 0;
          for (int k = 0; k < K; ++k) ref += fA[(m + shift) * KMAX + k] * fB[n * KMAX + k];
          if (ref != hD[m * N + n]) ++bad;
        }
      printf("SW%d base_offset %s shift %d: %s (%d bad of %d)\n", RB, mode ? "=(addr>>7)&7" : "=0", shift,
             bad ? "WRONG" : "exact", bad, 128 * N);
    }
  return 0;
}
