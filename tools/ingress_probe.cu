// Probe: per-SM operand ingress (L2 -> shared memory) by load method.
//   mode 0: TMA 2-D tiled, SW128, box 128 rows x 128 B (the conv kernel's B / pm-A loads)
//   mode 1: TMA 2-D tiled, no swizzle, box 64 rows x 256 B
//   mode 2: cp.async.bulk (1-D bulk copy) of 16 KB contiguous
//   mode 3: cp.async 16 B (LDGSTS) by 4 warps, 16 KB per stage
//   mode 4: mode 0 + mode 3 concurrently (TMA thread + 4 cp.async warps, halves each)
//   mode 5: TMA 2-D tiled SW128, box 256 rows x 64 B (SW64 rows)
// Each CTA streams its own region of a 96 MB buffer (L2 resident after warm-up).
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/ip tools/ingress_probe.cu -lcuda
#include <cuda.h>
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>

constexpr int STAGE = 16384, NST = 8, ITERS = 4096;
constexpr size_t REGION = 512 * 1024;   // bytes per CTA (re-read ITERS/32 times)

__device__ __forceinline__ void mbar_wait(uint32_t bar, uint32_t ph) {
  asm volatile("{\n.reg .pred P;\nW%=: mbarrier.try_wait.parity.shared::cta.b64 P, [%0], %1;\n@!P bra W%=;\n}" ::"r"(bar), "r"(ph) : "memory");
}

__global__ void __launch_bounds__(160, 1)
probe(const __grid_constant__ CUtensorMap m0, const __grid_constant__ CUtensorMap m1,
      const __grid_constant__ CUtensorMap m5, const __grid_constant__ CUtensorMap m4, const uint8_t *buf, int mode, long long *cyc) {
  extern __shared__ __align__(1024) uint8_t sm[];
  uint8_t *s = (uint8_t *)(((uintptr_t)sm + 1023) & ~(uintptr_t)1023);
  __shared__ __align__(8) uint64_t full[NST];
  const uint32_t sb = (uint32_t)__cvta_generic_to_shared(s);
  const int tid = threadIdx.x, warp = tid / 32;
  const size_t base = (size_t)blockIdx.x * REGION;
  const int rows_per_region = (int)(REGION / 128);
  if (tid == 0)
    for (int i = 0; i < NST; ++i) {
      asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"((uint32_t)__cvta_generic_to_shared(&full[i])));
    }
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  __syncthreads();
  long long t0 = clock64();
  if (mode <= 2 || mode == 5) {
    if (tid == 0) {
      for (int it = 0; it < ITERS; ++it) {
        const int st = it % NST;
        const uint32_t bar = (uint32_t)__cvta_generic_to_shared(&full[st]);
        if (it >= NST) mbar_wait(bar, ((it / NST) - 1) & 1);
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(STAGE) : "memory");
        const uint32_t dst = sb + st * STAGE;
        const int blk = it % (int)(REGION / STAGE);
        if (mode == 0) {
          const int row = blockIdx.x * rows_per_region + blk * 128;
          asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4}], [%2];"
                       ::"r"(dst), "l"((uint64_t)&m0), "r"(bar), "r"(0), "r"(row) : "memory");
        } else if (mode == 1) {
          const int row = blockIdx.x * (int)(REGION / 256) + blk * 64;
          asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4}], [%2];"
                       ::"r"(dst), "l"((uint64_t)&m1), "r"(bar), "r"(0), "r"(row) : "memory");
        } else if (mode == 5) {
          const int row = blockIdx.x * (int)(REGION / 64) + blk * 256;
          asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4}], [%2];"
                       ::"r"(dst), "l"((uint64_t)&m5), "r"(bar), "r"(0), "r"(row) : "memory");
        } else {
          asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                       ::"r"(dst), "l"(buf + base + (size_t)blk * STAGE), "r"(STAGE), "r"(bar) : "memory");
        }
      }
      for (int st = 0; st < NST; ++st) {
        const int last = ITERS - NST + st;
        mbar_wait((uint32_t)__cvta_generic_to_shared(&full[last % NST]), (last / NST) & 1);
      }
    }
  } else {
    // cp.async by warps 1..4 (mode 3: all bytes; mode 4: half, TMA thread the other half)
    const int half = mode == 4;
    if (warp >= 1) {
      const int t = tid - 32;           // 0..127
      const int bytes = half ? STAGE / 2 : STAGE;
      for (int it = 0; it < ITERS; ++it) {
        const int st = it % NST;
        const int blk = it % (int)(REGION / STAGE);
        const uint8_t *src = buf + base + (size_t)blk * STAGE + (half ? STAGE / 2 : 0);
        const uint32_t dst = sb + st * STAGE + (half ? STAGE / 2 : 0);
        for (int o = t * 16; o < bytes; o += 128 * 16)
          asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(dst + o), "l"(src + o) : "memory");
        asm volatile("cp.async.commit_group;" ::: "memory");
        asm volatile("cp.async.wait_group 6;" ::: "memory");
      }
      asm volatile("cp.async.wait_all;" ::: "memory");
    } else if (half && tid == 0) {
      for (int it = 0; it < ITERS; ++it) {
        const int st = it % NST;
        const uint32_t bar = (uint32_t)__cvta_generic_to_shared(&full[st]);
        if (it >= NST) mbar_wait(bar, ((it / NST) - 1) & 1);
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(STAGE / 2) : "memory");
        const int blk = it % (int)(REGION / STAGE);
        const int row = blockIdx.x * rows_per_region + blk * 128;
        asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4}], [%2];"
                     ::"r"(sb + st * STAGE), "l"((uint64_t)&m4), "r"(bar), "r"(0), "r"(row) : "memory");
      }
      for (int st = 0; st < NST; ++st) {
        const int last = ITERS - NST + st;
        mbar_wait((uint32_t)__cvta_generic_to_shared(&full[last % NST]), (last / NST) & 1);
      }
    }
  }
  __syncthreads();
  if (tid == 0) cyc[blockIdx.x] = clock64() - t0;
}

typedef CUresult (*EncFn)(CUtensorMap *, CUtensorMapDataType, cuuint32_t, void *, const cuuint64_t *,
                          const cuuint64_t *, const cuuint32_t *, const cuuint32_t *,
                          CUtensorMapInterleave, CUtensorMapSwizzle, CUtensorMapL2promotion,
                          CUtensorMapFloatOOBfill);

int main() {
  const int MAXG = 148;
  uint8_t *buf;
  long long *cyc;
  const size_t total = REGION * MAXG;
  cudaMalloc(&buf, total);
  cudaMemset(buf, 1, total);
  cudaMalloc(&cyc, MAXG * sizeof(long long));
  void *fp;
  cudaDriverEntryPointQueryResult q;
  cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fp, cudaEnableDefault, &q);
  EncFn enc = (EncFn)fp;
  CUtensorMap m0, m1, m5, m4;
  {
    cuuint64_t dims[2] = {64, total / 128}, str[1] = {128};
    cuuint32_t box[2] = {64, 64}, es[2] = {1, 1};
    CUresult r = enc(&m4, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, buf, dims, str, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
        CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    printf("enc m4 %d\n", (int)r);
  }
  {
    cuuint64_t dims[2] = {64, total / 128}, str[1] = {128};
    cuuint32_t box[2] = {64, 128}, es[2] = {1, 1};
    enc(&m0, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, buf, dims, str, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
        CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  }
  {
    cuuint64_t dims[2] = {128, total / 256}, str[1] = {256};
    cuuint32_t box[2] = {128, 64}, es[2] = {1, 1};
    printf("enc m1 %d\n", (int)enc(&m1, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, buf, dims, str, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
        CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE));
  }
  {
    cuuint64_t dims[2] = {32, total / 64}, str[1] = {64};
    cuuint32_t box[2] = {32, 256}, es[2] = {1, 1};
    enc(&m5, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, buf, dims, str, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
        CU_TENSOR_MAP_SWIZZLE_64B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  }
  const int smem = NST * STAGE + 1024;
  cudaFuncSetAttribute(probe, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  const char *names[] = {"TMA SW128 128x128B", "TMA noswz 64x256B", "bulk 1-D 16KB", "cp.async 4 warps",
                         "TMA + cp.async", "TMA SW64 256x64B"};
  for (int mode = 0; mode < 6; ++mode)
    for (int grid : {148, 74, 16}) {
      probe<<<grid, 160, smem>>>(m0, m1, m5, m4, buf, mode, cyc);   // warm
      cudaEvent_t e0, e1;
      cudaEventCreate(&e0);
      cudaEventCreate(&e1);
      cudaEventRecord(e0);
      probe<<<grid, 160, smem>>>(m0, m1, m5, m4, buf, mode, cyc);
      cudaEventRecord(e1);
      cudaError_t err = cudaDeviceSynchronize();
      if (err != cudaSuccess) { printf("mode %d: %s\n", mode, cudaGetErrorString(err)); return 1; }
      float ms;
      cudaEventElapsedTime(&ms, e0, e1);
      long long h[MAXG];
      cudaMemcpy(h, cyc, grid * sizeof(long long), cudaMemcpyDeviceToHost);
      double avg = 0;
      for (int i = 0; i < grid; ++i) avg += h[i];
      avg /= grid;
      const double bytes = (double)ITERS * STAGE;
      printf("%-20s grid %3d: %.1f B/cyc/SM, chip %.2f TB/s\n", names[mode], grid, bytes / avg,
             bytes * grid / (ms * 1e-3) / 1e12);
      fflush(stdout);
    }
  return 0;
}
