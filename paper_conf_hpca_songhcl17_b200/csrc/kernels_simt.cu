// kernels_simt.cu -- SIMT kernels of the hot path (sm_100a):
//   a1 input staging, final unstaging, FP32 implicit-GEMM conv/FC check path
//   (the paper's SGEMM), a4 LRN, a5 pooling, a7 softmax + entropy.
// Activations are NHWC; all arithmetic is fp32; storage is bf16 or fp32.
#include "budget.cuh"
#include "pcnn_internal.h"

namespace pcnn {

// ------------------------------------------------------------ small helpers
__device__ __forceinline__ float tf32_rna(float v) {
  unsigned r;
  asm("cvt.rna.tf32.f32 %0, %1;" : "=r"(r) : "f"(v));
  return __uint_as_float(r);
}

__device__ __forceinline__ float load_act(const void *p, int st, size_t i) {
  return st == ST_BF16 ? __bfloat162float(((const __nv_bfloat16 *)p)[i])
                       : ((const float *)p)[i];
}

__device__ __forceinline__ void store_act(void *p, int st, size_t i, float v,
                                          int tf32_round) {
  if (st == ST_BF16)
    ((__nv_bfloat16 *)p)[i] = __float2bfloat16_rn(v);
  else
    ((float *)p)[i] = tf32_round ? tf32_rna(v) : v;
}

// ------------------------------------------------------------ a1: staging
// One thread per (pixel, 4-channel group): reads NCHW (coalesced along W per
// channel), writes NHWC with zero-filled channel padding.
__global__ void stage_input_kernel(const float *__restrict__ x, void *y, int st,
                                   int B, int C, int H, int W, int Cs,
                                   int tf32_round) {
  const long long HW = (long long)H * W;
  const int groups4 = Cs / 4;
  const long long total = (long long)B * HW * groups4;
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < total;
       i += (long long)gridDim.x * blockDim.x) {
    const long long pix = i % (B * HW);
    const int cg = (int)(i / (B * HW));
    const long long n = pix / HW, hw = pix % HW;
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      const int c = cg * 4 + j;
      float v = 0.f;
      if (c < C) v = __ldg(&x[(n * C + c) * HW + hw]);
      store_act(y, st, (size_t)pix * Cs + c, v, tf32_round);
    }
  }
}

cudaError_t launch_stage_input(const float *x, void *y, int st, int B, int C,
                               int H, int W, int Cs, int tf32_round,
                               cudaStream_t s) {
  const long long total = (long long)B * H * W * (Cs / 4);
  int grid = (int)((total + 255) / 256);
  if (grid > 148 * 16) grid = 148 * 16;
  if (grid < 1) grid = 1;
  stage_input_kernel<<<grid, 256, 0, s>>>(x, y, st, B, C, H, W, Cs, tf32_round);
  return cudaGetLastError();
}

// final NHWC storage -> NCHW fp32 (C,H,W flatten order, reading R5)
__global__ void unstage_output_kernel(const void *x, int st, float *y, int B,
                                      int C, int H, int W, int Cs) {
  const long long HW = (long long)H * W;
  const long long total = (long long)B * C * HW;
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < total;
       i += (long long)gridDim.x * blockDim.x) {
    const long long n = i / (C * HW);
    const long long rem = i % (C * HW);
    const int c = (int)(rem / HW);
    const long long hw = rem % HW;
    y[i] = load_act(x, st, (size_t)((n * HW + hw) * Cs + c));
  }
}

cudaError_t launch_unstage_output(const void *x, int st, float *y, int B,
                                  int C, int H, int W, int Cs, cudaStream_t s) {
  const long long total = (long long)B * C * H * W;
  int grid = (int)((total + 255) / 256);
  if (grid > 148 * 16) grid = 148 * 16;
  if (grid < 1) grid = 1;
  unstage_output_kernel<<<grid, 256, 0, s>>>(x, st, y, B, C, H, W, Cs);
  return cudaGetLastError();
}

// ------------------------------------------------------------ FP32 SIMT conv
// Classic smem-tiled SGEMM (Volkov-Demmel style): a 64x64 sub-matrix
// of O per CTA, 256 threads x (4x4) micro-tiles, BK = 16.  The A tile is
// gathered straight from the NHWC activations (implicit im2col, Fig. 2 step 1
// never materialised).  Every output element sums its K terms in increasing
// k order, independent of tiling and budget.
constexpr int SB_M = 64, SB_N = 64, SB_K = 16;

int conv_simt_tiles(const ConvGeom &g) {
  return ((g.M + SB_M - 1) / SB_M) * ((g.Nfg + SB_N - 1) / SB_N) * g.groups;
}
void conv_simt_tile_shape(int *tm, int *tn) { *tm = SB_M; *tn = SB_N; }

__global__ void __launch_bounds__(256)
conv_simt_kernel(ConvGeom g, const float *__restrict__ x,
                 const float *__restrict__ w, const float *__restrict__ bias,
                 float *__restrict__ y, const int *__restrict__ ktab, Budget b,
                 int mtiles, int ntiles) {
  __shared__ float As[SB_K][SB_M + 4];
  __shared__ float Bs[SB_K][SB_N + 4];
  __shared__ long long row_base[SB_M];
  __shared__ int row_ih[SB_M], row_iw[SB_M];
  const int tid = threadIdx.x;
  const int tx = tid % 16, ty = tid / 16;
  const long long tiles = (long long)mtiles * ntiles * g.groups;
  const int HoWo = g.Ho * g.Wo;

  for_each_tile(b, tiles, [&](long long t) {
    const int mt = (int)(t % mtiles);
    const long long rest = t / mtiles;
    const int nt = (int)(rest % ntiles);
    const int grp = (int)(rest / ntiles);
    const int m0 = mt * SB_M, n0 = nt * SB_N;
    __syncthreads();
    if (tid < SB_M) {
      const int m = m0 + tid;
      if (m < g.M) {
        const int n = m / HoWo, pq = m % HoWo;
        const int p = pq / g.Wo, q = pq % g.Wo;
        row_base[tid] = (long long)n * g.H * g.W * g.Cs + (long long)grp * g.Cg;
        row_ih[tid] = p * g.stride - g.pad;
        row_iw[tid] = q * g.stride - g.pad;
      } else {
        row_base[tid] = -1;
        row_ih[tid] = 0;
        row_iw[tid] = 0;
      }
    }
    float acc[4][4];
#pragma unroll
    for (int i = 0; i < 4; ++i)
#pragma unroll
      for (int j = 0; j < 4; ++j) acc[i][j] = 0.f;
    __syncthreads();

    for (int k0 = 0; k0 < g.K; k0 += SB_K) {
#pragma unroll
      for (int i = 0; i < 4; ++i) {
        const int e = tid + 256 * i;
        const int kk = e % SB_K, row = e / SB_K;
        const int k = k0 + kk;
        float v = 0.f;
        const long long base = row_base[row];
        if (k < g.K && base >= 0) {
          int r = 0, s = 0, c = k;
          if (ktab) {
            const int e2 = __ldg(&ktab[k]);
            r = (e2 >> 24) & 0xFF;
            s = (e2 >> 16) & 0xFF;
            c = e2 & 0xFFFF;
          }
          const int ih = row_ih[row] + r, iw = row_iw[row] + s;
          if (ih >= 0 && ih < g.H && iw >= 0 && iw < g.W)
            v = __ldg(&x[base + ((long long)ih * g.W + iw) * g.Cs + c]);
        }
        As[kk][row] = v;
        const int ncol = n0 + row;
        float wv = 0.f;
        if (ncol < g.Nfg && k < g.K)
          wv = __ldg(&w[((long long)grp * g.Nfg + ncol) * g.Kpad + k]);
        Bs[kk][row] = wv;
      }
      __syncthreads();
#pragma unroll
      for (int kk = 0; kk < SB_K; ++kk) {
        float a[4], bb[4];
#pragma unroll
        for (int i = 0; i < 4; ++i) a[i] = As[kk][ty * 4 + i];
#pragma unroll
        for (int j = 0; j < 4; ++j) bb[j] = Bs[kk][tx * 4 + j];
#pragma unroll
        for (int i = 0; i < 4; ++i)
#pragma unroll
          for (int j = 0; j < 4; ++j) acc[i][j] = fmaf(a[i], bb[j], acc[i][j]);
      }
      __syncthreads();
    }
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      const int m = m0 + ty * 4 + i;
      if (m >= g.M) continue;
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        const int n = n0 + tx * 4 + j;
        if (n >= g.Nfg) continue;
        const int col = grp * g.Nfg + n;
        float v = acc[i][j] + (bias ? __ldg(&bias[col]) : 0.f);
        if (g.relu) v = fmaxf(v, 0.f);
        if (g.out_mode == OUT_F32_TF32) v = tf32_rna(v);
        y[(long long)m * g.out_cs + col] = v;
      }
    }
  });
}

int simt_conv_occupancy() {
  int n = 0;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n, conv_simt_kernel, 256, 0);
  return n > 0 ? n : 1;
}

cudaError_t launch_conv_simt(const ConvGeom &g, const float *x, const float *w,
                             const float *bias, float *y, const int *ktab,
                             const Budget &b, int grid, cudaStream_t s) {
  const int mtiles = (g.M + SB_M - 1) / SB_M;
  const int ntiles = (g.Nfg + SB_N - 1) / SB_N;
  conv_simt_kernel<<<grid, 256, 0, s>>>(g, x, w, bias, y, ktab, b, mtiles,
                                        ntiles);
  return cudaGetLastError();
}

// ------------------------------------------------------------ a4: LRN
// Across-channel LRN (reading R3) on NHWC: one warp per pixel; the pixel's
// channel vector is staged in smem and each lane sums its 5-channel window.
constexpr int LRN_WARPS = 8;
constexpr int LRN_MAXC = 1024;

__global__ void __launch_bounds__(LRN_WARPS * 32)
lrn_kernel(const void *x, void *y, int st, int tf32_round, long long pixels,
           int C, int size, float alpha, float beta, float k, Budget b) {
  __shared__ float buf[LRN_WARPS][LRN_MAXC];
  const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
  const int half = size / 2;
  const float a_over_n = alpha / (float)size;
  const long long tiles = (pixels + LRN_WARPS - 1) / LRN_WARPS;
  for_each_tile(b, tiles, [&](long long t) {
    const long long pix = t * LRN_WARPS + warp;
    if (pix < pixels) {
      const size_t base = (size_t)pix * C;
      for (int c = lane; c < C; c += 32) buf[warp][c] = load_act(x, st, base + c);
      __syncwarp();
      for (int c = lane; c < C; c += 32) {
        const int lo = c - half < 0 ? 0 : c - half;
        const int hi = c + half > C - 1 ? C - 1 : c + half;
        float sq = 0.f;
        for (int cc = lo; cc <= hi; ++cc) sq = fmaf(buf[warp][cc], buf[warp][cc], sq);
        const float scale = k + a_over_n * sq;
        store_act(y, st, base + c, buf[warp][c] * powf(scale, -beta), tf32_round);
      }
      __syncwarp();
    }
  });
}

int lrn_occupancy() {
  int n = 0;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n, lrn_kernel, LRN_WARPS * 32, 0);
  return n > 0 ? n : 1;
}

cudaError_t launch_lrn(const void *x, void *y, int st, int tf32_round,
                       long pixels, int C, int size, float alpha, float beta,
                       float k, const Budget &b, int grid, cudaStream_t s) {
  if (C > LRN_MAXC) return cudaErrorInvalidValue;
  lrn_kernel<<<grid, LRN_WARPS * 32, 0, s>>>(x, y, st, tf32_round, pixels, C,
                                             size, alpha, beta, k, b);
  return cudaGetLastError();
}

// ------------------------------------------------------------ a5: pooling
// One thread per (output pixel, channel); consecutive threads walk channels
// (contiguous in NHWC) so loads and stores are coalesced.
constexpr int POOL_THREADS = 256;

__global__ void __launch_bounds__(POOL_THREADS)
pool_kernel(const void *x, void *y, int st, int B, int H, int W, int C, int k,
            int stride, int Ho, int Wo, int is_max, int tf32_round, Budget b) {
  const long long total = (long long)B * Ho * Wo * C;
  const long long tiles = (total + POOL_THREADS - 1) / POOL_THREADS;
  for_each_tile(b, tiles, [&](long long t) {
    const long long i = t * POOL_THREADS + threadIdx.x;
    if (i < total) {
      const int c = (int)(i % C);
      const long long op = i / C;
      const int q = (int)(op % Wo);
      const long long np = op / Wo;
      const int p = (int)(np % Ho);
      const long long n = np / Ho;
      const int h0 = p * stride, w0 = q * stride;
      const int h1 = min(h0 + k, H), w1 = min(w0 + k, W);
      float m = -INFINITY, sum = 0.f;
      for (int h = h0; h < h1; ++h)
        for (int w = w0; w < w1; ++w) {
          const float v = load_act(x, st, (size_t)(((n * H + h) * W + w) * C + c));
          m = fmaxf(m, v);
          sum += v;
        }
      const float out = is_max ? m : sum / (float)(k * k);
      store_act(y, st, (size_t)i, out, is_max ? 0 : tf32_round);
    }
  });
}

int pool_occupancy() {
  int n = 0;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n, pool_kernel, POOL_THREADS, 0);
  return n > 0 ? n : 1;
}

cudaError_t launch_pool(const void *x, void *y, int st, int B, int H, int W,
                        int C, int k, int stride, int Ho, int Wo, int is_max,
                        int tf32_round, const Budget &b, int grid,
                        cudaStream_t s) {
  pool_kernel<<<grid, POOL_THREADS, 0, s>>>(x, y, st, B, H, W, C, k, stride, Ho,
                                            Wo, is_max, tf32_round, b);
  return cudaGetLastError();
}

// ------------------------------------------------------------ a7: softmax + entropy
// One warp per image: max and sum by warp shuffles (eq. 2).
// H = ln S - sum_j p_j (z_j - max), algebraically -sum p ln p (reading R6).
__global__ void softmax_entropy_kernel(const float *__restrict__ z, float *p,
                                       float *h, int B, int N) {
  const int warp = (blockIdx.x * blockDim.x + threadIdx.x) / 32;
  const int lane = threadIdx.x % 32;
  if (warp >= B) return;
  const float *zr = z + (size_t)warp * N;
  float m = -INFINITY;
  for (int j = lane; j < N; j += 32) m = fmaxf(m, zr[j]);
  for (int o = 16; o; o >>= 1) m = fmaxf(m, __shfl_xor_sync(0xffffffffu, m, o));
  float s = 0.f, sz = 0.f;
  for (int j = lane; j < N; j += 32) {
    const float d = zr[j] - m;
    const float e = expf(d);
    s += e;
    sz += e * d;
  }
  for (int o = 16; o; o >>= 1) {
    s += __shfl_xor_sync(0xffffffffu, s, o);
    sz += __shfl_xor_sync(0xffffffffu, sz, o);
  }
  const float inv = 1.f / s;
  if (p)
    for (int j = lane; j < N; j += 32) p[(size_t)warp * N + j] = expf(zr[j] - m) * inv;
  if (h && lane == 0) h[warp] = logf(s) - sz * inv;
}

cudaError_t launch_softmax_entropy(const float *z, float *p, float *h, int B,
                                   int N, cudaStream_t s) {
  const int warps_per_block = 8;
  const int grid = (B + warps_per_block - 1) / warps_per_block;
  softmax_entropy_kernel<<<grid, warps_per_block * 32, 0, s>>>(z, p, h, B, N);
  return cudaGetLastError();
}

}  // namespace pcnn
