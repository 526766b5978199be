// kernels_simt.cu -- SIMT kernels of the hot path (sm_100a):
//   a1 input staging (incl. space-to-depth), final unstaging, FP32 implicit-GEMM
//   conv/FC check path
//   (the paper's SGEMM), a4/a5 LRN + pooling (fused), a7 softmax + entropy.
// Activations are NHWC; all arithmetic is fp32; storage is bf16 or fp32.
#include <cstdlib>
#include <algorithm>

#include "budget.cuh"
#include "lrn_math.cuh"
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

// ------------------------------------------------------------ vector helpers
// 16 B of storage = 8 bf16 or 4 fp32 values, converted to / from fp32.
template <int ST>
struct Vec16 {
  static constexpr int N = ST == ST_BF16 ? 8 : 4;
  float v[N];
  __device__ __forceinline__ void load(const void *p) { from_raw(*(const uint4 *)p); }
  __device__ __forceinline__ void from_raw(const uint4 raw) {
    if constexpr (ST == ST_BF16) {
      // bf16 -> fp32 is a 16-bit shift of the bit pattern (exact)
      const uint32_t w[4] = {raw.x, raw.y, raw.z, raw.w};
#pragma unroll
      for (int i = 0; i < 4; ++i) {
        v[2 * i] = __uint_as_float(w[i] << 16);
        v[2 * i + 1] = __uint_as_float(w[i] & 0xFFFF0000u);
      }
    } else {
      const float *f = (const float *)&raw;
#pragma unroll
      for (int i = 0; i < 4; ++i) v[i] = f[i];
    }
  }
  __device__ __forceinline__ void store(void *p, int tf32_round) const {
    uint4 raw;
    if constexpr (ST == ST_BF16) {
      __nv_bfloat162 *h = (__nv_bfloat162 *)&raw;
#pragma unroll
      for (int i = 0; i < 4; ++i) h[i] = __floats2bfloat162_rn(v[2 * i], v[2 * i + 1]);
    } else {
      float *f = (float *)&raw;
#pragma unroll
      for (int i = 0; i < 4; ++i) f[i] = tf32_round ? tf32_rna(v[i]) : v[i];
    }
    *(uint4 *)p = raw;
  }
};

// ------------------------------------------------------------ a1: staging
// NCHW fp32 -> NHWC storage [B][Hs][Ws][Cs].  Output channel c' < blk^2*C is
// (dr, ds, c) = (c' / C / blk, c' / C % blk, c' % C) and reads input pixel
// (h'*blk - pad + dr, w'*blk - pad + ds); blk = 1 is the plain layout with
// zero channel padding, blk = stride is space-to-depth for a strided first
// conv (turns AlexNet's 11x11/4 conv on 3 channels into a 3x3/1 conv on 48,
// so the GEMM's K is 432 instead of 968 with 8-channel padding).  Rounded to
// the storage precision (BF16 RN-even, TF32 RN-away).  One thread per
// (pixel, 16 B chunk); chunk index fastest so the stores are coalesced.
template <int ST>
__global__ void __launch_bounds__(256)
stage_input_kernel(const float *__restrict__ x, void *y, int B, int C, int H, int W, int Hs,
                   int Ws, int Cs, int blk, int pad, int tf32_round) {
  pdl_enter();   // PDL: wait for the previous kernel, let the next one launch
  constexpr int VN = Vec16<ST>::N;
  const int chunks = Cs / VN;
  const long long total = (long long)B * Hs * Ws * chunks;
  const long long HW = (long long)H * W;
  const int creal = blk * blk * C;
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < total;
       i += (long long)gridDim.x * blockDim.x) {
    const int ch = (int)(i % chunks);
    const long long pix = i / chunks;
    const int ws = (int)(pix % Ws);
    const long long t = pix / Ws;
    const int hs = (int)(t % Hs);
    const long long n = t / Hs;
    Vec16<ST> o;
#pragma unroll
    for (int j = 0; j < VN; ++j) {
      const int cp = ch * VN + j;
      float v = 0.f;
      if (cp < creal) {
        const int b = cp / C, c = cp - b * C;
        const int ih = hs * blk - pad + b / blk, iw = ws * blk - pad + b % blk;
        if (ih >= 0 && ih < H && iw >= 0 && iw < W) v = __ldg(&x[(n * C + c) * HW + (long long)ih * W + iw]);
      }
      o.v[j] = v;
    }
    o.store((char *)y + (size_t)i * 16, tf32_round);
  }
}

// Row-staged variant: one CTA per (image, output row).  The blk input rows
// x C channels it needs are loaded into smem with coalesced (consecutive-W)
// reads, then every (pixel, 16 B chunk) of the output row is assembled from
// smem and stored coalesced.  Used when those rows fit in 48 KB.
template <int ST>
__global__ void __launch_bounds__(256)
stage_rows_kernel(const float *__restrict__ x, void *y, int C, int H, int W, int Hs, int Ws,
                  int Cs, int blk, int pad, int tf32_round) {
  pdl_enter();   // PDL: wait for the previous kernel, let the next one launch
  extern __shared__ float rows[];                  // [blk][C][W] then the channel map
  constexpr int VN = Vec16<ST>::N;
  const int hs = blockIdx.x % Hs;
  const long long n = blockIdx.x / Hs;
  const long long HW = (long long)H * W;
  const int nrow = blk * C;
  int *cmap = (int *)(rows + nrow * W);            // [Cs]: row offset | column delta
  // 4 B cp.async keeps every load of the staged rows in flight
  const uint32_t sbase = (uint32_t)__cvta_generic_to_shared(rows);
  for (int i = threadIdx.x; i < nrow * W; i += blockDim.x) {
    const int rc = i / W, w = i - rc * W;          // rc = dr * C + c
    const int dr = rc / C, c = rc - dr * C;
    const int ih = hs * blk - pad + dr;
    const bool ok = ih >= 0 && ih < H;
    const float *src = ok ? x + (n * C + c) * HW + (long long)ih * W + w : x;
    asm volatile("cp.async.ca.shared.global [%0], [%1], 4, %2;" ::"r"(sbase + 4u * i),
                 "l"(src), "r"(ok ? 4 : 0)
                 : "memory");
  }
  const int creal = blk * blk * C;
  for (int cp = threadIdx.x; cp < Cs; cp += blockDim.x) {
    if (cp < creal) {
      const int b = cp / C, c = cp - b * C;
      cmap[cp] = (((b / blk) * C + c) * W) << 4 | (b % blk);   // row base, ds
    } else {
      cmap[cp] = -1;
    }
  }
  asm volatile("cp.async.commit_group;\ncp.async.wait_all;" ::: "memory");
  __syncthreads();
  const int chunks = Cs / VN;
  char *yrow = (char *)y + ((size_t)(n * Hs + hs) * Ws) * Cs * (ST == ST_BF16 ? 2 : 4);
  for (int i = threadIdx.x; i < Ws * chunks; i += blockDim.x) {
    const int ws = i / chunks, ch = i - ws * chunks;
    const int iw0 = ws * blk - pad;
    Vec16<ST> o;
#pragma unroll
    for (int j = 0; j < VN; ++j) {
      const int e = cmap[ch * VN + j];
      float v = 0.f;
      if (e >= 0) {
        const int iw = iw0 + (e & 15);
        if (iw >= 0 && iw < W) v = rows[(e >> 4) + iw];
      }
      o.v[j] = v;
    }
    o.store(yrow + (size_t)i * 16, tf32_round);
  }
}

// Specialised staging for the networks' 3-channel inputs: one CTA per
// (image, output row), one thread per output pixel.  The BLK input rows x 3
// channels are staged in smem with a 16 B-aligned row pitch, each thread reads
// its BLK x BLK x 3 window as float4s (BLK = 4, space-to-depth) or scalars
// (BLK = 1) and writes its whole Cs-channel pixel with 16 B stores.
template <int ST, int BLK>
__global__ void __launch_bounds__(256)
stage_c3_kernel(const float *__restrict__ x, void *y, int H, int W, int Hs, int Ws, int Cs,
                int pad, int tf32_round) {
  pdl_enter();   // PDL: wait for the previous kernel, let the next one launch
  constexpr int C = 3;
  constexpr int VN = Vec16<ST>::N;
  constexpr int ESZ = ST == ST_BF16 ? 2 : 4;
  extern __shared__ float rows[];                  // [BLK][C][Wp]
  const int Wp = ((Ws * BLK + 3) & ~3) + 4;        // covers iw in [-pad, Ws*BLK)
  const int hs = blockIdx.x % Hs;
  const long long n = blockIdx.x / Hs;
  const long long HW = (long long)H * W;
  const uint32_t sbase = (uint32_t)__cvta_generic_to_shared(rows);
  // smem column j holds input column j - pad
  for (int i = threadIdx.x; i < BLK * C * Wp; i += blockDim.x) {
    const int rc = i / Wp, j = i - rc * Wp;
    const int dr = rc / C, c = rc - dr * C;
    const int ih = hs * BLK - pad + dr, iw = j - pad;
    const bool ok = ih >= 0 && ih < H && iw >= 0 && iw < W;
    const float *src = ok ? x + (n * C + c) * HW + (long long)ih * W + iw : x;
    asm volatile("cp.async.ca.shared.global [%0], [%1], 4, %2;" ::"r"(sbase + 4u * i),
                 "l"(src), "r"(ok ? 4 : 0)
                 : "memory");
  }
  asm volatile("cp.async.commit_group;\ncp.async.wait_all;" ::: "memory");
  __syncthreads();
  char *yrow = (char *)y + ((size_t)(n * Hs + hs) * Ws) * Cs * ESZ;
  for (int ws = threadIdx.x; ws < Ws; ws += blockDim.x) {
    float v[BLK * BLK * C];                          // channel cp = (dr*BLK + ds)*C + c
#pragma unroll
    for (int dr = 0; dr < BLK; ++dr)
#pragma unroll
      for (int c = 0; c < C; ++c) {
        const float *rp = rows + (dr * C + c) * Wp + ws * BLK;
        if constexpr (BLK == 4) {
          const float4 q = *(const float4 *)rp;
          v[(dr * BLK + 0) * C + c] = q.x;
          v[(dr * BLK + 1) * C + c] = q.y;
          v[(dr * BLK + 2) * C + c] = q.z;
          v[(dr * BLK + 3) * C + c] = q.w;
        } else {
#pragma unroll
          for (int ds = 0; ds < BLK; ++ds) v[(dr * BLK + ds) * C + c] = rp[ds];
        }
      }
    char *py = yrow + (size_t)ws * Cs * ESZ;
    constexpr int NREAL = BLK * BLK * C;
    constexpr int MAXCH = (NREAL + VN - 1) / VN + 8;   // stored channels <= NREAL + padding
#pragma unroll
    for (int ch = 0; ch < MAXCH; ++ch) {
      if (ch * VN >= Cs) break;
      Vec16<ST> o;
#pragma unroll
      for (int j = 0; j < VN; ++j) o.v[j] = ch * VN + j < NREAL ? v[ch * VN + j] : 0.f;
      o.store(py + ch * 16, tf32_round);
    }
  }
}

// First-layer im2col staging (3-channel inputs, S x S taps, stride st, pad):
// output pixel (n, p, q) gets the K = S*S*3 values of its receptive field in
// (r, s, c) order, zero-padded to Kp channels, so the first conv runs as a
// 1x1 conv with one full 128 B TMA slab per pixel.  One CTA per output row;
// the S input rows x 3 channels are staged in smem with cp.async.
template <int ST, int S>
__global__ void __launch_bounds__(256)
stage_im2col_kernel(const float *__restrict__ x, void *y, int H, int W, int Ho, int Wo, int Kp,
                    int st, int pad, int halo, int tf32_round) {
  pdl_enter();   // PDL: wait for the previous kernel, let the next one launch
  constexpr int C = 3, K = S * S * C;
  constexpr int VN = Vec16<ST>::N;
  constexpr int ESZ = ST == ST_BF16 ? 2 : 4;
  extern __shared__ float rows[];                  // [S][C][Wp], column j = input col j - pad
  const int Wp = (Wo - 1) * st + S;
  const int p = blockIdx.x % Ho;
  const long long n = blockIdx.x / Ho;
  const long long HW = (long long)H * W;
  const uint32_t sbase = (uint32_t)__cvta_generic_to_shared(rows);
  for (int i = threadIdx.x; i < S * C * Wp; i += blockDim.x) {
    const int rc = i / Wp, j = i - rc * Wp;
    const int r = rc / C, c = rc - r * C;
    const int ih = p * st - pad + r, iw = j - pad;
    const bool ok = ih >= 0 && ih < H && iw >= 0 && iw < W;
    const float *src = ok ? x + (n * C + c) * HW + (long long)ih * W + iw : x;
    asm volatile("cp.async.ca.shared.global [%0], [%1], 4, %2;" ::"r"(sbase + 4u * i),
                 "l"(src), "r"(ok ? 4 : 0)
                 : "memory");
  }
  asm volatile("cp.async.commit_group;\ncp.async.wait_all;" ::: "memory");
  __syncthreads();
  // rows of a zero-haloed output grid (Ho + halo) x (Wo + halo) (shared
  // halo layout, interior at the origin): the interior only (the consumer
  // never reads the halo rows of a 1x1 conv)
  const int Wop = Wo + halo;
  char *yrow = (char *)y + ((size_t)(n * (Ho + halo) + p) * Wop) * Kp * ESZ;
  for (int q = threadIdx.x; q < Wo; q += blockDim.x) {
    float v[K];
#pragma unroll
    for (int r = 0; r < S; ++r)
#pragma unroll
      for (int s2 = 0; s2 < S; ++s2)
#pragma unroll
        for (int c = 0; c < C; ++c) v[(r * S + s2) * C + c] = rows[(r * C + c) * Wp + q * st + s2];
    char *py = yrow + (size_t)q * Kp * ESZ;
    constexpr int MAXCH = (K + VN - 1) / VN + 16;
#pragma unroll
    for (int ch = 0; ch < MAXCH; ++ch) {
      if (ch * VN >= Kp) break;
      Vec16<ST> o;
#pragma unroll
      for (int j = 0; j < VN; ++j) o.v[j] = ch * VN + j < K ? v[ch * VN + j] : 0.f;
      o.store(py + ch * 16, tf32_round);
    }
  }
}

// 3-channel first-layer staging, both layouts (a1): output pixel (h, w) of
// an output row, channel k < K = D*D*3 is input (c, h*step - pad + a,
// w*step - pad + b) with k = (a*D + b)*3 + c -- the (dr, ds, c) order of
// space-to-depth (D = step = blk) and the (r, s, c) order of first-layer
// im2col (D = S, step = conv stride) -- and 0 for K <= k < Kp.  One CTA per
// (image, band of output rows): the band's input rows x 3 channels are copied
// to smem as aligned 16 B chunks (the fp32 rows are not 16 B aligned: each
// keeps its 0..3-float shift), then each thread assembles one 16 B output
// chunk of a pixel -- its chunk's channel map is fixed and lives in registers.
template <int ST>
__global__ void __launch_bounds__(256)
stage_gather3_kernel(const float *__restrict__ x, void *y, int B, int H, int W, int Ho, int Wo,
                     int Kp, int D, int step, int pad, int halo, int rows_per_cta, int tf32_round) {
  pdl_enter();   // PDL: wait for the previous kernel, let the next one launch
  constexpr int C = 3;
  constexpr int VN = Vec16<ST>::N;
  extern __shared__ __align__(16) float g3_rows[];   // [span*C][Wrow] input rows, 16 B-aligned copies
  const int Wrow = (W + 3) / 4 * 4 + 4;              // room for the 0..3 float alignment shift
  const int cpr = Wrow / 4;                          // 16 B chunks loaded per row
  const int K = D * D * C;
  const int bands = (Ho + rows_per_cta - 1) / rows_per_cta;
  const int max_rows = ((rows_per_cta - 1) * step + D) * C;
  // this thread's output chunk is fixed (blockDim % chunks == 0), so its
  // channel -> (row, column offset) map is computed once, outside the
  // persistent band loop
  const int chunks = Kp / VN;
  const int ch = threadIdx.x % chunks;
  int rr[VN], bb[VN];
#pragma unroll
  for (int e = 0; e < VN; ++e) {
    const int k = ch * VN + e;
    if (k < K) {
      const int ab = k / C, c = k - ab * C;
      const int a = ab / D;
      rr[e] = a * C + c;
      bb[e] = ab - a * D - pad;
    } else {
      rr[e] = -1;
      bb[e] = 0;
    }
  }
  for (long long t = blockIdx.x; t < (long long)B * bands; t += gridDim.x) {
  const int h0 = (int)(t % bands) * rows_per_cta;
  const int nh = min(rows_per_cta, Ho - h0);
  const long long n = t / bands;
  const int span = (nh - 1) * step + D;
  const int nrow = span * C;
  __syncthreads();   // the previous band's rows are no longer read
  int *row_shift = (int *)(g3_rows + (size_t)max_rows * Wrow);   // -1: row outside the image
  const long long total = (long long)B * C * H * W;
  // phase 1: each input row [ih][0, W) of the band as aligned 16 B chunks
  // (cp.async, zero fill past the end of the tensor); shift = row start % 4
  const float inv_cpr = 1.f / (float)cpr;
  const uint32_t sbase = (uint32_t)__cvta_generic_to_shared(g3_rows);
  for (int v = threadIdx.x; v < nrow * cpr; v += blockDim.x) {
    int r, jc;
    fdivmod(v, cpr, inv_cpr, r, jc);
    const int a = r / C, c = r - a * C;
    const int ih = h0 * step - pad + a;
    if (ih < 0 || ih >= H) continue;
    const long long e0 = ((n * C + c) * H + ih) * (long long)W;
    const long long a0 = e0 & ~3LL;
    const long long e = a0 + 4LL * jc;
    const int bytes = e + 4 <= total ? 16 : (e < total ? (int)(total - e) * 4 : 0);
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;" ::"r"(
                     sbase + (uint32_t)((r * Wrow + 4 * jc) * 4)),
                 "l"(x + (bytes ? e : 0)), "r"(bytes)
                 : "memory");
  }
  for (int r = threadIdx.x; r < nrow; r += blockDim.x) {
    const int a = r / C, c = r - a * C;
    const int ih = h0 * step - pad + a;
    row_shift[r] = (ih < 0 || ih >= H) ? -1 : (int)((((n * C + c) * H + ih) * (long long)W) & 3);
  }
  asm volatile("cp.async.commit_group;\ncp.async.wait_all;" ::: "memory");
  __syncthreads();
  // phase 2: thread = (pixel, 16 B output chunk)
  const int Wop = Wo + halo;                         // shared-halo output grid
  const int ppi = blockDim.x / chunks;               // pixels per pass
  for (int hh = 0; hh < nh; ++hh) {
    const int h = h0 + hh;
    char *yrow = (char *)y + ((size_t)(n * (Ho + halo) + h) * Wop) *
                                 (size_t)Kp * (ST == ST_BF16 ? 2 : 4);
    // per channel of this thread's chunk: smem index of input column 0 of its
    // row in this output row, minus the pad (can be negative: the sentinel for
    // a row outside the image is NOROW)
    constexpr int NOROW = -(1 << 30);
    int base[VN];
#pragma unroll
    for (int e = 0; e < VN; ++e) {
      base[e] = NOROW;
      if (rr[e] >= 0) {
        const int r = rr[e] + hh * step * C;
        const int sh = row_shift[r];
        if (sh >= 0) base[e] = r * Wrow + sh + bb[e];
      }
    }
    for (int w = threadIdx.x / chunks; w < Wo; w += ppi) {
      const int iw0 = w * step - pad;                // column of tap offset 0
      const bool inner = iw0 >= 0 && iw0 + D <= W;
      Vec16<ST> o;
#pragma unroll
      for (int e = 0; e < VN; ++e) {
        float val = 0.f;
        if (base[e] != NOROW) {
          const int iw = w * step + bb[e];
          if (inner || (iw >= 0 && iw < W)) val = g3_rows[base[e] + w * step];
        }
        o.v[e] = val;
      }
      o.store(yrow + ((size_t)w * chunks + ch) * 16, tf32_round);
    }
  }
  }   // bands
}

static bool gather3_ok(int st, int W, int Kp, int D, int step) {
  const int vn = st == ST_BF16 ? 8 : 4;
  const int Wrow = (W + 3) / 4 * 4 + 4;
  return Kp % vn == 0 && 256 % (Kp / vn) == 0 && D * D * 3 <= Kp &&
         (size_t)D * 3 * (Wrow * sizeof(float) + sizeof(int)) <= 96 * 1024 && step >= 1;
}

static cudaError_t launch_gather3(const float *x, void *y, int st, int B, int H, int W, int Ho,
                                  int Wo, int Kp, int D, int step, int pad, int halo,
                                  int tf32_round, cudaStream_t s) {
  static const int rows_env = [] {
    const char *e = exp_env("PCNN_STAGE_ROWS");
    return e ? atoi(e) : 0;
  }();
  const int vn = st == ST_BF16 ? 8 : 4;
  if (Kp % vn || 256 % (Kp / vn) || D * D * 3 > Kp) return cudaErrorInvalidValue;
  const int Wrow = (W + 3) / 4 * 4 + 4;
  auto smem_for = [&](int R) {
    return (size_t)((R - 1) * step + D) * 3 * (Wrow * sizeof(float) + sizeof(int));
  };
  int R = rows_env > 0 ? rows_env : 1;
  if (rows_env <= 0)
    while (R < 8 && R < Ho && smem_for(R + 1) <= 40 * 1024) ++R;
  const size_t smem = smem_for(R);
  if (smem > 96 * 1024) return cudaErrorInvalidValue;
  const long long tiles = (long long)B * ((Ho + R - 1) / R);
  // persistent CTAs: a full wave of resident CTAs walks the bands
  int occ = 1;
  if (st == ST_BF16)
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, stage_gather3_kernel<ST_BF16>, 256, smem);
  else
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, stage_gather3_kernel<ST_F32>, 256, smem);
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  const unsigned grid = (unsigned)std::min<long long>(tiles, (long long)sms * std::max(occ, 1));
  if (st == ST_BF16) {
    if (smem > 48 * 1024)
      cudaFuncSetAttribute(stage_gather3_kernel<ST_BF16>,
                           cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    launch_pdl(stage_gather3_kernel<ST_BF16>, dim3(grid), dim3(256), smem, s, x, y, B, H, W, Ho, Wo, Kp, D, step,
                                                           pad, halo, R, 0);
  } else {
    if (smem > 48 * 1024)
      cudaFuncSetAttribute(stage_gather3_kernel<ST_F32>,
                           cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    launch_pdl(stage_gather3_kernel<ST_F32>, dim3(grid), dim3(256), smem, s, x, y, B, H, W, Ho, Wo, Kp, D, step,
                                                          pad, halo, R, tf32_round);
  }
  return cudaGetLastError();
}

// Warp-cooperative bulk staging of input rows for the first-layer staging
// kernels: rows [row0, row0 + nrows) of the C channels of image n (row lr =
// a * C + c at buf + lr * pitch), one bulk TMA copy per row of its 16 B-aligned
// superset, one row per lane.  sh[lr] = the row's start offset in floats, -1
// for rows outside the image (read as zeros).  The bytes are announced after
// the copies (the mbarrier tx-count may go negative within a phase; the phase
// cannot complete before lane 0's arrive).  Rows whose superset would run
// past the tensor are loaded with plain loads.
__device__ __forceinline__ void bulk_rows(const float *__restrict__ x, uintptr_t xend,
                                          long long n, int C, int H, int W, int row0,
                                          int nrows, float *buf, int *sh, int pitch,
                                          uint32_t bar) {
  const int lane = threadIdx.x & 31;
  uint32_t bytes = 0;
  for (int lr = lane; lr < nrows * C; lr += 32) {
    const int a = lr / C, c = lr - a * C, ih = row0 + a;
    if (ih < 0 || ih >= H) {
      sh[lr] = -1;
      continue;
    }
    const uintptr_t src = (uintptr_t)(x + ((size_t)(n * C + c) * H + ih) * W);
    const uintptr_t a0 = src & ~(uintptr_t)15;
    const uint32_t nb = (uint32_t)(((src + (uintptr_t)W * 4 - a0) + 15) & ~(uintptr_t)15);
    float *dst = buf + (size_t)lr * pitch;
    if (a0 + nb > xend) {
      for (int j = 0; j < W; ++j) dst[j] = __ldg((const float *)src + j);
      sh[lr] = 0;
      continue;
    }
    sh[lr] = (int)((src - a0) >> 2);
    bytes += nb;
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
        ::"r"((uint32_t)__cvta_generic_to_shared(dst)), "l"(a0), "r"(nb), "r"(bar)
        : "memory");
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) bytes += __shfl_xor_sync(0xffffffffu, bytes, o);
  __syncwarp();
  if (lane == 0)
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes)
                 : "memory");
}

__device__ __forceinline__ void mbar_wait_parity(uint32_t bar, uint32_t par) {
  asm volatile(
      "{\n.reg .pred P1;\nW_%=:\nmbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n"
      "@!P1 bra W_%=;\n}\n" ::"r"(bar), "r"(par)
      : "memory");
}

// First-layer im2col staging for 3-channel inputs, S x S taps, stride 1,
// pad S/2 (VGG conv1_1): persistent CTAs over bands of R output rows; the
// band's R + S - 1 input rows per channel arrive by bulk TMA copies (two
// buffers); one thread per output pixel gathers its S*S*3 values (rows
// re-aligned by their start offset, zeros outside the image) in (r, s, c)
// order, zero-pads to Kp channels and writes the pixel with 16 B stores into
// the interior of the halo-h output grid.
template <int ST, int S>
__global__ void __launch_bounds__(256)
stage_im2c3_kernel(const float *__restrict__ x, void *y, int B, int H, int W, int Kp, int halo,
                   int R, int tf32_round) {
  pdl_enter();   // PDL: wait for the previous kernel, let the next one launch
  constexpr int C = 3, PAD = S / 2, NREAL = S * S * C;
  constexpr int VN = Vec16<ST>::N;
  constexpr int ESZ = ST == ST_BF16 ? 2 : 4;
  extern __shared__ __align__(128) uint8_t ic_smem[];
  const int pitch = ((W + 3) / 4 + 1) * 4;
  const int rows = (R + S - 1) * C;
  float *bufs = (float *)ic_smem;
  uint64_t *bar = (uint64_t *)(ic_smem + (size_t)2 * rows * pitch * 4);
  int *shift = (int *)(bar + 2);
  const int bands = (H + R - 1) / R;
  const long long tiles = (long long)B * bands;
  const uintptr_t xend = (uintptr_t)(x + (size_t)B * C * H * W);
  const uint32_t bar0 = (uint32_t)__cvta_generic_to_shared(bar);
  const int Hp = H + halo, Wp = W + halo;        // shared-halo output grid
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(bar0));
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(bar0 + 8));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  auto issue = [&](long long t, int b) {
    const long long n = t / bands;
    const int p0 = (int)(t % bands) * R, nh = min(R, H - p0);
    bulk_rows(x, xend, n, C, H, W, p0 - PAD, nh + S - 1, bufs + (size_t)b * rows * pitch,
              shift + b * rows, pitch, bar0 + 8 * b);
  };
  long long t = blockIdx.x;
  if (threadIdx.x < 32 && t < tiles) issue(t, 0);
  uint32_t phase[2] = {0, 0};
  for (int b = 0; t < tiles; t += gridDim.x, b ^= 1) {
    if (threadIdx.x < 32 && t + gridDim.x < tiles) issue(t + gridDim.x, b ^ 1);
    mbar_wait_parity(bar0 + 8 * b, phase[b]);
    phase[b] ^= 1;
    const long long n = t / bands;
    const int p0 = (int)(t % bands) * R, nh = min(R, H - p0);
    const float *buf = bufs + (size_t)b * rows * pitch;
    const int *sh = shift + b * rows;
    for (int pix = threadIdx.x; pix < nh * W; pix += blockDim.x) {
      const int hr = pix / W, q = pix - hr * W;
      float v[NREAL];                               // channel (r * S + s) * C + c
#pragma unroll
      for (int r = 0; r < S; ++r)
#pragma unroll
        for (int c = 0; c < C; ++c) {
          const int lr = (hr + r) * C + c, o = sh[lr];
          const float *rp = buf + (size_t)lr * pitch + o;
#pragma unroll
          for (int s2 = 0; s2 < S; ++s2) {
            const int col = q + s2 - PAD;
            v[(r * S + s2) * C + c] = (o >= 0 && col >= 0 && col < W) ? rp[col] : 0.f;
          }
        }
      char *py = (char *)y + ((((size_t)n * Hp + p0 + hr) * Wp + q) * (size_t)Kp) * ESZ;
      constexpr int NCH = (NREAL + VN - 1) / VN;
#pragma unroll
      for (int ch = 0; ch < NCH; ++ch) {
        Vec16<ST> o;
#pragma unroll
        for (int j = 0; j < VN; ++j) o.v[j] = ch * VN + j < NREAL ? v[ch * VN + j] : 0.f;
        o.store(py + ch * 16, tf32_round);
      }
      for (int ch = NCH; ch < Kp / VN; ++ch) *(uint4 *)(py + ch * 16) = make_uint4(0, 0, 0, 0);
    }
    __syncthreads();
  }
}

cudaError_t launch_stage_im2col(const float *x, void *y, int st, int B, int C, int H, int W,
                                int S, int stride, int pad, int Ho, int Wo, int Kp,
                                int halo, int tf32_round, cudaStream_t s) {
  if (C != 3 || (S != 3 && S != 5)) return cudaErrorInvalidValue;
  if (!exp_env("PCNN_OLD_STAGE") && S == 3 && stride == 1 && pad == 1 && Ho == H && Wo == W &&
      Kp >= 27 && Kp % (st == ST_BF16 ? 8 : 4) == 0) {
    const int R = 2;
    const int pitch = ((W + 3) / 4 + 1) * 4;
    const size_t smem = (size_t)2 * (R + 2) * 3 * pitch * 4 + 16 + 2 * (R + 2) * 3 * 4;
    if (smem <= 200 * 1024) {
      const long long tiles = (long long)B * ((H + R - 1) / R);
      int dev = 0, sms = 148, occ = 1;
      cudaGetDevice(&dev);
      cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
#define PCNN_IC3(STT)                                                                          \
  do {                                                                                         \
    if (smem > 48 * 1024)                                                                      \
      cudaFuncSetAttribute(stage_im2c3_kernel<STT, 3>,                                         \
                           cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);            \
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, stage_im2c3_kernel<STT, 3>, 256, smem); \
    const unsigned grid = (unsigned)std::min<long long>(tiles, (long long)sms * std::max(occ, 1)); \
    launch_pdl(stage_im2c3_kernel<STT, 3>, dim3(grid), dim3(256), smem, s, x, y, B, H, W, Kp, halo, R, tf32_round); \
  } while (0)
      if (st == ST_BF16) PCNN_IC3(ST_BF16);
      else PCNN_IC3(ST_F32);
#undef PCNN_IC3
      return cudaGetLastError();
    }
  }
  if (!exp_env("PCNN_OLD_STAGE") && gather3_ok(st, W, Kp, S, stride))
    return launch_gather3(x, y, st, B, H, W, Ho, Wo, Kp, S, stride, pad, halo, tf32_round, s);
  const size_t smem = (size_t)S * C * ((Wo - 1) * stride + S) * sizeof(float);
  if (smem > 48 * 1024) return cudaErrorInvalidValue;
  const unsigned grid = (unsigned)((long long)B * Ho);
#define PCNN_IM2COL(STT, SS) \
  launch_pdl(stage_im2col_kernel<STT, SS>, dim3(grid), dim3(256), smem, s, x, y, H, W, Ho, Wo, Kp, stride, pad, halo, tf32_round)
  if (st == ST_BF16) {
    if (S == 3) PCNN_IM2COL(ST_BF16, 3); else PCNN_IM2COL(ST_BF16, 5);
  } else {
    if (S == 3) PCNN_IM2COL(ST_F32, 3); else PCNN_IM2COL(ST_F32, 5);
  }
#undef PCNN_IM2COL
  return cudaGetLastError();
}

// Band kernels (staging, LRN + pool) shorten their bands at small batches
// until a launch has about two CTAs per SM.
constexpr long long kBandTargetCtas = 2 * 148;

// Space-to-depth staging for 3-channel inputs, block 4, no padding (AlexNet
// conv1 11x11/4 -> 3x3/1 on 48 channels).  A persistent CTA walks bands of R
// staged rows; one thread copies each needed input row (all W floats of one
// channel) into shared memory with a single bulk TMA copy of its 16 B-aligned
// superset, the next band's copies in flight while the current band is
// converted (two buffers, one mbarrier each).  Then one thread per staged
// pixel reads its 4 x 3 row segments as 16 B vectors (re-aligned by the row's
// start offset), permutes them into the (dr, ds, c) channel order and writes
// the whole pixel (Cs channels, zero padded) with 16 B stores.
#ifndef PCNN_S2D_MINB
#define PCNN_S2D_MINB 1
#endif
#ifndef PCNN_S2D_ROWS_DEFAULT
#define PCNN_S2D_ROWS_DEFAULT 4
#endif
#ifndef PCNN_S2D_NBUF
#define PCNN_S2D_NBUF 2
#endif

template <int ST>
__global__ void __launch_bounds__(256, PCNN_S2D_MINB)
stage_s2d4_kernel(const float *__restrict__ x, void *y, int B, int H, int W, int Hs, int Ws,
                  int Cs, int R, int tf32_round) {
  pdl_enter();   // PDL: wait for the previous kernel, let the next one launch
  constexpr int C = 3, BLK = 4;
  constexpr int VN = Vec16<ST>::N;
  constexpr int ESZ = ST == ST_BF16 ? 2 : 4;
  extern __shared__ __align__(128) uint8_t s2_smem[];
  const int pitch = ((W + 3) / 4 + 1) * 4;            // floats per smem row (16 B multiple)
  const int rows = R * BLK * C;
  constexpr int NB = PCNN_S2D_NBUF;                   // band buffers in flight
  float *bufs = (float *)s2_smem;                     // [NB][rows][pitch]
  uint64_t *bar = (uint64_t *)(s2_smem + (size_t)NB * rows * pitch * 4);
  int *shift = (int *)(bar + NB);                     // [NB][rows]: start offset, -1 = zero row
  const int bands = (Hs + R - 1) / R;
  const long long tiles = (long long)B * bands;
  const uintptr_t xend = (uintptr_t)(x + (size_t)B * C * H * W);
  const uint32_t bar0 = (uint32_t)__cvta_generic_to_shared(bar);
  if (threadIdx.x == 0) {
#pragma unroll
    for (int i = 0; i < NB; ++i) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(bar0 + 8 * i));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  auto issue = [&](long long t, int b) {
    const long long n = t / bands;
    const int h0 = (int)(t % bands) * R, nh = min(R, Hs - h0);
    bulk_rows(x, xend, n, C, H, W, h0 * BLK, nh * BLK, bufs + (size_t)b * rows * pitch,
              shift + b * rows, pitch, bar0 + 8 * b);
  };
  long long t = blockIdx.x;
  if (threadIdx.x < 32)
    for (int i = 0; i < NB - 1; ++i)
      if (t + (long long)i * gridDim.x < tiles) issue(t + (long long)i * gridDim.x, i);
  uint32_t phase[NB] = {};
  for (int b = 0; t < tiles; t += gridDim.x, b = b + 1 == NB ? 0 : b + 1) {
    {   // the band NB - 1 tiles ahead goes into the buffer freed last iteration
      const long long ta = t + (long long)(NB - 1) * gridDim.x;
      const int ba = (b + NB - 1) % NB;
      if (threadIdx.x < 32 && ta < tiles) issue(ta, ba);
    }
    {
      const uint32_t bb = bar0 + 8 * b, par = phase[b];
      asm volatile(
          "{\n.reg .pred P1;\nW_%=:\nmbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n"
          "@!P1 bra W_%=;\n}\n" ::"r"(bb), "r"(par)
          : "memory");
      phase[b] ^= 1;
    }
    const long long n = t / bands;
    const int h0 = (int)(t % bands) * R, nh = min(R, Hs - h0);
    const float *buf = bufs + (size_t)b * rows * pitch;
    const int *sh = shift + b * rows;
    for (int p = threadIdx.x; p < nh * Ws; p += blockDim.x) {
      const int hr = p / Ws, ws = p - hr * Ws;
      float v[BLK * BLK * C];                       // channel (dr * BLK + ds) * C + c
#pragma unroll
      for (int dr = 0; dr < BLK; ++dr)
#pragma unroll
        for (int c = 0; c < C; ++c) {
          const int lr = (hr * BLK + dr) * C + c;
          const int o = sh[lr];
          float q[4] = {0.f, 0.f, 0.f, 0.f};
          if (o >= 0) {
            const float *rp = buf + (size_t)lr * pitch + ws * BLK;
            const float4 lo = *(const float4 *)rp;
            const float4 hi = *(const float4 *)(rp + 4);
            const float w8[8] = {lo.x, lo.y, lo.z, lo.w, hi.x, hi.y, hi.z, hi.w};
#pragma unroll
            for (int ds = 0; ds < 4; ++ds) {
              float val = w8[ds];
              val = o == 1 ? w8[ds + 1] : val;
              val = o == 2 ? w8[ds + 2] : val;
              val = o == 3 ? w8[ds + 3] : val;
              q[ds] = ws * BLK + ds < W ? val : 0.f;
            }
          }
#pragma unroll
          for (int ds = 0; ds < BLK; ++ds) v[(dr * BLK + ds) * C + c] = q[ds];
        }
      char *py = (char *)y + (((size_t)n * Hs + h0 + hr) * Ws + ws) * (size_t)Cs * ESZ;
      constexpr int NREAL = BLK * BLK * C;
      constexpr int NCH = (NREAL + VN - 1) / VN;      // chunks holding real channels
#pragma unroll
      for (int ch = 0; ch < NCH; ++ch) {
        Vec16<ST> o;
#pragma unroll
        for (int j = 0; j < VN; ++j) o.v[j] = ch * VN + j < NREAL ? v[ch * VN + j] : 0.f;
        o.store(py + ch * 16, tf32_round);
      }
      for (int ch = NCH; ch < Cs / VN; ++ch) *(uint4 *)(py + ch * 16) = make_uint4(0, 0, 0, 0);
    }
    __syncthreads();   // buffer b is refilled by the next-but-one band
  }
}

static cudaError_t launch_stage_s2d4(const float *x, void *y, int st, int B, int H, int W,
                                     int Hs, int Ws, int Cs, int tf32_round, cudaStream_t s) {
  static const int R3 = [] {                         // staged rows per band
    const char *e = exp_env("PCNN_S2D_ROWS");
    return e && atoi(e) > 0 ? atoi(e) : PCNN_S2D_ROWS_DEFAULT;
  }();
  int R = R3;                                        // small batches: shorter bands
  while (R > 1 && (long long)B * ((Hs + R - 1) / R) < kBandTargetCtas) --R;
  const int pitch = ((W + 3) / 4 + 1) * 4;
  const size_t smem = (size_t)PCNN_S2D_NBUF * (R * 12 * pitch * 4 + 8 + R * 12 * 4);
  if (smem > 200 * 1024) return cudaErrorInvalidValue;
  const long long tiles = (long long)B * ((Hs + R - 1) / R);
  int dev = 0, sms = 148, occ = 1;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
#define PCNN_S2D(STT)                                                                          \
  do {                                                                                         \
    if (smem > 48 * 1024)                                                                      \
      cudaFuncSetAttribute(stage_s2d4_kernel<STT>, cudaFuncAttributeMaxDynamicSharedMemorySize, \
                           (int)smem);                                                         \
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, stage_s2d4_kernel<STT>, 256, smem);    \
    const unsigned grid = (unsigned)std::min<long long>(tiles, (long long)sms * std::max(occ, 1)); \
    launch_pdl(stage_s2d4_kernel<STT>, dim3(grid), dim3(256), smem, s, x, y, B, H, W, Hs, Ws, Cs, R, tf32_round);  \
  } while (0)
  if (st == ST_BF16) PCNN_S2D(ST_BF16);
  else PCNN_S2D(ST_F32);
#undef PCNN_S2D
  return cudaGetLastError();
}

cudaError_t launch_stage_input(const float *x, void *y, int st, int B, int C, int H, int W,
                               int Hs, int Ws, int Cs, int blk, int pad, int tf32_round,
                               cudaStream_t s) {
  const char *old_stage = exp_env("PCNN_OLD_STAGE");   // A/B: the staged-gather kernels
  if (C == 3 && blk == 4 && pad == 0 && !old_stage && Cs >= 48 &&
      Cs % (st == ST_BF16 ? 8 : 4) == 0 && Hs * 4 <= H + 3 && Ws * 4 <= W + 3)
    return launch_stage_s2d4(x, y, st, B, H, W, Hs, Ws, Cs, tf32_round, s);
  if (C == 3 && !old_stage && gather3_ok(st, W, Cs, blk, blk))
    return launch_gather3(x, y, st, B, H, W, Hs, Ws, Cs, blk, blk, pad, 0, tf32_round, s);
  if (C == 3 && (blk == 4 || blk == 1) && W <= 4096) {
    const int Wp = ((Ws * blk + 3) & ~3) + 4;
    const size_t smem = (size_t)blk * C * Wp * sizeof(float);
    const unsigned grid = (unsigned)((long long)B * Hs);
    if (smem <= 48 * 1024) {
      if (st == ST_BF16) {
        if (blk == 4)
          launch_pdl(stage_c3_kernel<ST_BF16, 4>, dim3(grid), dim3(256), smem, s, x, y, H, W, Hs, Ws, Cs, pad, 0);
        else
          launch_pdl(stage_c3_kernel<ST_BF16, 1>, dim3(grid), dim3(256), smem, s, x, y, H, W, Hs, Ws, Cs, pad, 0);
      } else {
        if (blk == 4)
          launch_pdl(stage_c3_kernel<ST_F32, 4>, dim3(grid), dim3(256), smem, s, x, y, H, W, Hs, Ws, Cs, pad, tf32_round);
        else
          launch_pdl(stage_c3_kernel<ST_F32, 1>, dim3(grid), dim3(256), smem, s, x, y, H, W, Hs, Ws, Cs, pad, tf32_round);
      }
      return cudaGetLastError();
    }
  }
  const size_t rows_bytes = (size_t)blk * C * W * sizeof(float) + (size_t)Cs * sizeof(int);
  if (rows_bytes <= 48 * 1024 && blk <= 15) {
    const long long grid = (long long)B * Hs;
    if (st == ST_BF16)
      launch_pdl(stage_rows_kernel<ST_BF16>, dim3((unsigned)grid), dim3(256), rows_bytes, s, x, y, C, H, W, Hs, Ws,
                                                                          Cs, blk, pad, 0);
    else
      launch_pdl(stage_rows_kernel<ST_F32>, dim3((unsigned)grid), dim3(256), rows_bytes, s, x, y, C, H, W, Hs, Ws,
                                                                         Cs, blk, pad, tf32_round);
    return cudaGetLastError();
  }
  const int vn = st == ST_BF16 ? 8 : 4;
  const long long total = (long long)B * Hs * Ws * (Cs / vn);
  const int grid = (int)std::max<long long>(1, std::min<long long>((total + 255) / 256, 148 * 16));
  if (st == ST_BF16)
    launch_pdl(stage_input_kernel<ST_BF16>, dim3(grid), dim3(256), 0, s, x, y, B, C, H, W, Hs, Ws, Cs, blk, pad, 0);
  else
    launch_pdl(stage_input_kernel<ST_F32>, dim3(grid), dim3(256), 0, s, x, y, B, C, H, W, Hs, Ws, Cs, blk, pad,
                                                    tf32_round);
  return cudaGetLastError();
}

// pcnn_infer_host_u8: uint8 NCHW pixels -> fp32 network input
// (pixel - mean[c]) * scale, 16 pixels per thread (one 16 B load, four 16 B
// stores).  HW % 16 == 0 takes the vector path; else one pixel per step.
__global__ void pixels_u8_kernel(const unsigned char *__restrict__ px, const float *__restrict__ mean,
                                 float scale, float *__restrict__ y, long long total, int C, int HW) {
  pdl_enter();   // PDL: wait for the previous kernel, let the next one launch
  const long long stride = (long long)gridDim.x * blockDim.x;
  if ((HW & 15) == 0) {
    for (long long v = blockIdx.x * (long long)blockDim.x + threadIdx.x; v < total / 16; v += stride) {
      const long long e = v * 16;
      const int c = (int)((e / HW) % C);
      const float m = mean[c];
      const uint4 raw = __ldg((const uint4 *)(px + e));
      const uint32_t w[4] = {raw.x, raw.y, raw.z, raw.w};
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        float4 o;
        o.x = ((float)(w[q] & 0xFF) - m) * scale;
        o.y = ((float)((w[q] >> 8) & 0xFF) - m) * scale;
        o.z = ((float)((w[q] >> 16) & 0xFF) - m) * scale;
        o.w = ((float)(w[q] >> 24) - m) * scale;
        *(float4 *)(y + e + 4 * q) = o;
      }
    }
    return;
  }
  for (long long e = blockIdx.x * (long long)blockDim.x + threadIdx.x; e < total; e += stride)
    y[e] = ((float)px[e] - mean[(e / HW) % C]) * scale;
}

cudaError_t launch_pixels_u8(const unsigned char *px, const float *mean, float scale, float *y,
                             int B, int C, int HW, cudaStream_t s) {
  const long long total = (long long)B * C * HW;
  const long long work = (HW & 15) == 0 ? total / 16 : total;
  const int grid = (int)std::max<long long>(1, std::min<long long>((work + 255) / 256, 148LL * 8));
  launch_pdl(pixels_u8_kernel, dim3(grid), dim3(256), 0, s, px, mean, scale, y, total, C, HW);
  return cudaGetLastError();
}

// final NHWC storage -> NCHW fp32 flatten (C,H,W order, reading R5)
__global__ void unstage_output_kernel(const void *x, int st, float *y, int B,
                                      int C, int H, int W, int Cs) {
  pdl_enter();   // PDL: wait for the previous kernel, let the next one launch
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
  launch_pdl(unstage_output_kernel, dim3(grid), dim3(256), 0, s, x, st, y, B, C, H, W, Cs);
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
  pdl_enter();   // PDL: wait for the previous kernel, let the next one launch
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
  launch_pdl(conv_simt_kernel, dim3(grid), dim3(256), 0, s, g, x, w, bias, y, ktab, b, mtiles,
                                        ntiles);
  return cudaGetLastError();
}

// ------------------------------------------------------------ a4 + a5: LRN and pooling
// One kernel for LRN (reading R3), max / avg pooling (R4), and the fused
// LRN -> max-pool pair of AlexNet (norm1 -> pool1, norm2 -> pool2).  NHWC.
// A tile is (image n, output row p, output columns [q0, q0 + Q)): the pool
// window rows [p*s, p*s + k) x the columns they cover are contiguous runs of
// C channels in memory, loaded into smem with coalesced 16 B vectors.  LRN
// (when enabled) transforms every staged pixel's channel vector -- rounded to
// the storage precision exactly as the stand-alone layer would store it -- and
// the pool reduces k x k windows of 16 B channel chunks.  Without pooling
// (k = s = 1) the kernel is the stand-alone LRN; without LRN it is the pool.
struct LrnPoolArgs {
  const void *x;
  void *y;
  int B, H, W, C;
  int lrn_size;            // 0 = no LRN
  float lrn_alpha_over_n, lrn_beta, lrn_k;
  int k, s, is_max;        // pool window / stride (1, 1 = no pool)
  int Ho, Wo;
  int Q, nqt;              // output columns per tile, tiles per row
  int tf32_round;
  int Cout;                // stored output channels
  int ocg, ocp;            // output group layout: ocg real channels padded to
                           // ocp per group (0 = compact, Cout == C)
  int hi, ho;              // zero halo of the input / output layout: shared-halo grids
                           // [H + h][W + h], interior at the origin
  int R, nbands;           // band kernel: output rows per tile, bands per image
  Budget b;
};

template <int ST, int LS>
__global__ void __launch_bounds__(256) lrn_pool_kernel(const LrnPoolArgs a) {
  pdl_enter();   // PDL: wait for the previous kernel, let the next one launch
  extern __shared__ __align__(16) uint8_t lp_smem[];
  constexpr int ESZ = ST == ST_BF16 ? 2 : 4;
  constexpr int VN = Vec16<ST>::N;
  const int C = a.C, chunks = C / VN;
  const int wc_max = (a.Q - 1) * a.s + a.k;
  const size_t tile_elems = (size_t)a.k * wc_max * C;
  uint8_t *T = lp_smem;                                  // staged input
  uint8_t *U = LS > 0 ? lp_smem + tile_elems * ESZ : lp_smem;   // LRN output
  const long long tiles = (long long)a.B * a.Ho * a.nqt;
  const float inv_chunks = 1.f / (float)chunks;

  for_each_tile(a.b, tiles, [&](long long t) {
    const int qt = (int)(t % a.nqt);
    const long long r2 = t / a.nqt;
    const int p = (int)(r2 % a.Ho);
    const long long n = r2 / a.Ho;
    const int q0 = qt * a.Q, q1 = min(q0 + a.Q, a.Wo);
    const int h0 = p * a.s, h1 = min(h0 + a.k, a.H);
    const int w0 = q0 * a.s, w1 = min((q1 - 1) * a.s + a.k, a.W);
    const int nr = h1 - h0, wc = w1 - w0;
    // shared-halo layouts ([H + h][W + h], interior at the origin, the zero
    // rows / columns after it)
    const int Hp = a.H + a.hi, Wp = a.W + a.hi;          // stored input grid
    const int Hop = a.Ho + a.ho, Wop = a.Wo + a.ho;      // stored output grid
    if (a.ho > 0) {
      // halo output: the last row's first tile zeroes the bottom halo rows,
      // the last column tile of every row that row's right halo columns
      const int oc16 = a.Cout * ESZ / 16;
      const uint4 z = make_uint4(0, 0, 0, 0);
      uint4 *yb = (uint4 *)a.y;
      if (qt == 0 && p == a.Ho - 1) {
        const size_t base = ((size_t)n * Hop + a.Ho) * Wop * oc16;
        for (int v = threadIdx.x; v < a.ho * Wop * oc16; v += blockDim.x) yb[base + v] = z;
      }
      const size_t rowb = ((size_t)n * Hop + p) * Wop * oc16;
      if (qt == a.nqt - 1)
        for (int v = threadIdx.x; v < a.ho * oc16; v += blockDim.x)
          yb[rowb + (size_t)a.Wo * oc16 + v] = z;
    }
    __syncthreads();
    // stage rows [h0, h1) x cols [w0, w1): each row segment is contiguous;
    // cp.async keeps every 16 B load of the tile in flight at once
    const int vec_per_row = wc * chunks;
    const float inv_vpr = 1.f / (float)vec_per_row;
    const uint32_t tbase = (uint32_t)__cvta_generic_to_shared(T);
    for (int v = threadIdx.x; v < nr * vec_per_row; v += blockDim.x) {
      int r, rem;
      fdivmod(v, vec_per_row, inv_vpr, r, rem);
      const size_t src = (((size_t)n * Hp + h0 + r) * Wp + w0) * C + (size_t)rem * VN;
      const uint32_t dst = tbase + (uint32_t)(((size_t)r * wc_max * C + (size_t)rem * VN) * ESZ);
      asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(dst),
                   "l"((const char *)a.x + src * ESZ)
                   : "memory");
    }
    asm volatile("cp.async.commit_group;\ncp.async.wait_all;" ::: "memory");
    __syncthreads();
    if (LS > 0) {
      // each thread: one 16 B channel chunk of one staged pixel; the window
      // needs HALF channels of the neighbouring chunks, read as whole vectors
      constexpr int HALF = LS / 2;
      static_assert(HALF <= VN, "LRN window wider than one neighbouring chunk");
      // walk every staged pixel slot (row pitch wc_max; unused slots are
      // harmless) so only one divmod by `chunks` is needed
      for (int v = threadIdx.x; v < nr * wc_max * chunks; v += blockDim.x) {
        int pix, ch;
        fdivmod(v, chunks, inv_chunks, pix, ch);
        const int r = 0, col = pix;
        const uint8_t *px = T + ((size_t)r * wc_max + col) * C * ESZ;
        Vec16<ST> prev, cur, next;
        cur.load(px + (size_t)ch * 16);
        if (ch > 0) prev.load(px + (size_t)(ch - 1) * 16);
        else
#pragma unroll
          for (int j = 0; j < VN; ++j) prev.v[j] = 0.f;
        if (ch + 1 < chunks) next.load(px + (size_t)(ch + 1) * 16);
        else
#pragma unroll
          for (int j = 0; j < VN; ++j) next.v[j] = 0.f;
        float sq[VN + 2 * HALF];
#pragma unroll
        for (int j = 0; j < VN + 2 * HALF; ++j) {
          const int t = j - HALF;            // channel offset from the chunk start
          const float xv = t < 0 ? prev.v[VN + t] : (t < VN ? cur.v[t] : next.v[t - VN]);
          sq[j] = __fmul_rn(xv, xv);
        }
        Vec16<ST> out;
        lrn_normalise<ST == ST_BF16, LS, VN>(sq, cur.v, a.lrn_k, a.lrn_alpha_over_n, a.lrn_beta,
                                             out.v);
        out.store(U + ((size_t)r * wc_max + col) * C * ESZ + (size_t)ch * 16, a.tf32_round);
      }
      __syncthreads();
    }
    // pool the staged (and normalised) rows; output chunk oc maps to input
    // chunk ch through the (optional) per-group channel padding
    const float inv = 1.f / (float)(a.k * a.k);
    const int ochunks = a.Cout / VN;
    const float inv_oc = 1.f / (float)ochunks;
    const int grp_real = a.ocg / VN, grp_pad = a.ocp / VN;
    for (int v = threadIdx.x; v < (q1 - q0) * ochunks; v += blockDim.x) {
      int qq, oc;
      fdivmod(v, ochunks, inv_oc, qq, oc);
      const int q = q0 + qq;
      int ch = oc;
      bool pad = false;
      if (grp_pad > 0) {
        const int gi = oc / grp_pad, j = oc - gi * grp_pad;
        pad = j >= grp_real;
        ch = gi * grp_real + j;
      }
      Vec16<ST> acc, cur;
#pragma unroll
      for (int j = 0; j < VN; ++j) acc.v[j] = pad ? 0.f : (a.is_max ? -INFINITY : 0.f);
      char *dst = (char *)a.y + ((((size_t)n * Hop + p) * Wop + q) * a.Cout + oc * VN) * ESZ;
      if (ST == ST_BF16 && a.is_max && !pad) {
        // max is exact in bf16: compare packed pairs, no conversions
        const int cs = q * a.s - w0, ce = min(cs + a.k, wc);
        __nv_bfloat162 m[4];
        const __nv_bfloat162 ninf = __float2bfloat162_rn(-INFINITY);
#pragma unroll
        for (int j = 0; j < 4; ++j) m[j] = ninf;
        for (int r = 0; r < nr; ++r)
          for (int col = cs; col < ce; ++col) {
            const uint4 raw = *(const uint4 *)(U + (((size_t)r * wc_max + col) * C + ch * VN) * ESZ);
            const __nv_bfloat162 *h = (const __nv_bfloat162 *)&raw;
#pragma unroll
            for (int j = 0; j < 4; ++j) m[j] = __hmax2(m[j], h[j]);
          }
        *(uint4 *)dst = *(const uint4 *)m;
        continue;
      }
      if (!pad) {
        const int cs = q * a.s - w0, ce = min(cs + a.k, wc);
        for (int r = 0; r < nr; ++r)
          for (int col = cs; col < ce; ++col) {
            cur.load(U + (((size_t)r * wc_max + col) * C + ch * VN) * ESZ);
#pragma unroll
            for (int j = 0; j < VN; ++j)
              acc.v[j] = a.is_max ? fmaxf(acc.v[j], cur.v[j]) : acc.v[j] + cur.v[j];
          }
        if (!a.is_max)
#pragma unroll
          for (int j = 0; j < VN; ++j) acc.v[j] *= inv;
      }
      acc.store(dst, a.is_max ? 0 : a.tf32_round);
    }
  });
}

// LRN (+ optional pool) over bands of R output rows: the band's input rows
// are staged once (cp.async, padded pixel pitch so per-pixel accesses are
// conflict-free), normalised IN PLACE by one thread per pixel streaming its
// channels in order (the 5-channel window of chunk j needs only the original
// tail of chunk j-1, kept in registers, and the head of chunk j+1, not yet
// overwritten), then pooled from smem.  Every input pixel is normalised once
// per band (rows shared by two bands: (R*s + k - s) / (R*s) recompute) instead
// of once per pooling window.  Same per-element arithmetic as lrn_pool_kernel
// and the conv epilogue (lrn_normalise), so results are identical.
template <int ST, int LS>
__global__ void __launch_bounds__(256) lrn_band_kernel(const LrnPoolArgs a) {
  pdl_enter();   // PDL: wait for the previous kernel, let the next one launch
  extern __shared__ __align__(16) uint8_t lb_smem[];
  constexpr int ESZ = ST == ST_BF16 ? 2 : 4;
  constexpr int VN = Vec16<ST>::N;
  constexpr int HALF = LS / 2;
  static_assert(HALF <= VN, "LRN window wider than one neighbouring chunk");
  const int C = a.C, chunks = C / VN;
  const int pitch = C * ESZ + 16;
  const long long tiles = (long long)a.B * a.nbands;
  const int Hp = a.H + a.hi, Wp = a.W + a.hi;             // shared-halo grids
  const int Hop = a.Ho + a.ho, Wop = a.Wo + a.ho;
  const float inv_chunks = 1.f / (float)chunks;

  for_each_tile(a.b, tiles, [&](long long t) {
    const int band = (int)(t % a.nbands);
    const long long n = t / a.nbands;
    const int p0 = band * a.R, p1 = min(p0 + a.R, a.Ho);
    const int h0 = p0 * a.s, h1 = min((p1 - 1) * a.s + a.k, a.H);
    const int nr = h1 - h0;
    if (a.ho > 0) {
      // zero the output halo cells this band owns: top / bottom halo rows
      // with the first / last band, left / right columns of its rows
      const int oc16 = a.Cout * ESZ / 16;
      const uint4 z = make_uint4(0, 0, 0, 0);
      uint4 *yb = (uint4 *)a.y;
      if (p1 == a.Ho)                    // bottom halo rows
        for (int v = threadIdx.x; v < a.ho * Wop * oc16; v += blockDim.x)
          yb[((size_t)n * Hop + a.Ho) * Wop * oc16 + v] = z;
      for (int v = threadIdx.x; v < (p1 - p0) * a.ho * oc16; v += blockDim.x) {   // right columns
        const int rr = v / (a.ho * oc16), o = v - rr * a.ho * oc16;
        const size_t rowb = ((size_t)n * Hop + p0 + rr) * Wop * oc16;
        yb[rowb + (size_t)a.Wo * oc16 + o] = z;
      }
    }
    __syncthreads();   // the previous band's pooling is done with smem
    const uint32_t sbase = (uint32_t)__cvta_generic_to_shared(lb_smem);
    const int npix = nr * a.W;
    for (int v = threadIdx.x; v < npix * chunks; v += blockDim.x) {
      int pix, ch;
      fdivmod(v, chunks, inv_chunks, pix, ch);
      const int r = pix / a.W, col = pix - r * a.W;
      const size_t src = (((size_t)n * Hp + h0 + r) * Wp + col) * C + (size_t)ch * VN;
      asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(
                       sbase + (uint32_t)(pix * pitch + ch * 16)),
                   "l"((const char *)a.x + src * ESZ)
                   : "memory");
    }
    asm volatile("cp.async.commit_group;\ncp.async.wait_all;" ::: "memory");
    __syncthreads();
    if (LS > 0) {
      for (int pix = threadIdx.x; pix < npix; pix += blockDim.x) {
        uint8_t *px = lb_smem + pix * pitch;
        float tail[HALF > 0 ? HALF : 1];
#pragma unroll
        for (int j = 0; j < HALF; ++j) tail[j] = 0.f;
        Vec16<ST> cur, nxt;
        cur.load(px);
        for (int ch = 0; ch < chunks; ++ch) {
          if (ch + 1 < chunks) nxt.load(px + (ch + 1) * 16);
          else
#pragma unroll
            for (int j = 0; j < VN; ++j) nxt.v[j] = 0.f;
          float sq[VN + 2 * HALF];
#pragma unroll
          for (int j = 0; j < VN + 2 * HALF; ++j) {
            const int o = j - HALF;
            const float xv = o < 0 ? tail[HALF + o] : (o < VN ? cur.v[o] : nxt.v[o - VN]);
            sq[j] = __fmul_rn(xv, xv);
          }
          Vec16<ST> out;
          lrn_normalise<ST == ST_BF16, LS, VN>(sq, cur.v, a.lrn_k, a.lrn_alpha_over_n,
                                               a.lrn_beta, out.v);
          out.store(px + ch * 16, a.tf32_round);
#pragma unroll
          for (int j = 0; j < HALF; ++j) tail[j] = cur.v[VN - HALF + j];
          cur = nxt;
        }
      }
      __syncthreads();
    }
    // pool (k = s = 1: copy) the normalised rows
    const float inv = 1.f / (float)(a.k * a.k);
    const int ochunks = a.Cout / VN;
    const float inv_oc = 1.f / (float)ochunks;
    const int grp_real = a.ocg / VN, grp_pad = a.ocp / VN;
    const int nq = a.Wo * ochunks;
    for (int v = threadIdx.x; v < (p1 - p0) * nq; v += blockDim.x) {
      const int rr = v / nq;
      int q, oc;
      fdivmod(v - rr * nq, ochunks, inv_oc, q, oc);
      const int pp = p0 + rr;
      int ch = oc;
      bool pad = false;
      if (grp_pad > 0) {
        const int gi = oc / grp_pad, j = oc - gi * grp_pad;
        pad = j >= grp_real;
        ch = gi * grp_real + j;
      }
      char *dst = (char *)a.y + ((((size_t)n * Hop + pp) * Wop + q) * a.Cout + oc * VN) * ESZ;
      const int rs = pp * a.s - h0, re = min(rs + a.k, nr);
      const int cs = q * a.s, ce = min(cs + a.k, a.W);
      if (ST == ST_BF16 && a.is_max) {
        __nv_bfloat162 m[4];
        const __nv_bfloat162 ninf = __float2bfloat162_rn(-INFINITY);
        const __nv_bfloat162 zero = __float2bfloat162_rn(0.f);
#pragma unroll
        for (int j = 0; j < 4; ++j) m[j] = pad ? zero : ninf;
        if (!pad)
          for (int r = rs; r < re; ++r)
            for (int col = cs; col < ce; ++col) {
              const uint4 raw = *(const uint4 *)(lb_smem + (r * a.W + col) * pitch + ch * 16);
              const __nv_bfloat162 *h = (const __nv_bfloat162 *)&raw;
#pragma unroll
              for (int j = 0; j < 4; ++j) m[j] = __hmax2(m[j], h[j]);
            }
        *(uint4 *)dst = *(const uint4 *)m;
        continue;
      }
      Vec16<ST> acc, cur;
#pragma unroll
      for (int j = 0; j < VN; ++j) acc.v[j] = pad ? 0.f : (a.is_max ? -INFINITY : 0.f);
      if (!pad) {
        for (int r = rs; r < re; ++r)
          for (int col = cs; col < ce; ++col) {
            cur.load(lb_smem + (r * a.W + col) * pitch + ch * 16);
#pragma unroll
            for (int j = 0; j < VN; ++j)
              acc.v[j] = a.is_max ? fmaxf(acc.v[j], cur.v[j]) : acc.v[j] + cur.v[j];
          }
        if (!a.is_max)
#pragma unroll
          for (int j = 0; j < VN; ++j) acc.v[j] *= inv;
      }
      acc.store(dst, a.is_max ? 0 : a.tf32_round);
    }
  });
}

// LRN (+ optional pool) over bands of R output rows, LRN in registers.
// P lanes of one warp share a pixel, each owning CPT consecutive 16 B channel
// chunks that it loads straight from global memory (a warp reads one
// contiguous run of pixels); the 2 channels of the window that lie in the
// neighbouring lanes' chunks come by warp shuffle, so there is no staging
// pass and no serial walk along the channels.  The normalised band is written
// once to shared memory (chunk c of pixel x at slot c ^ ((x*P + c/8) & 7) when
// CPT == 8, so neither the writes nor the pooling reads conflict) and pooled
// from there.  Same per-element arithmetic as the other LRN paths (sum order,
// lrn_normalise), so the results are identical.
template <int ST, int CPT, int MINB = 0>
__global__ void __launch_bounds__(256, MINB) lrn_reg_kernel(const LrnPoolArgs a) {
  pdl_enter();   // PDL: wait for the previous kernel, let the next one launch
  extern __shared__ __align__(16) uint8_t lr_smem[];
  constexpr int ESZ = ST == ST_BF16 ? 2 : 4;
  constexpr int VN = Vec16<ST>::N;
  constexpr int HALF = 2;                      // LRN size 5
  constexpr bool SWZ = CPT == 8;
  const int C = a.C, chunks = C / VN, P = chunks / CPT;
  const int lp = __ffs(P) - 1;                 // P is a power of two (lrn_reg_cpt)
  const float inv_w = 1.f / (float)a.W;
  const long long tiles = (long long)a.B * a.nbands;
  const int Hp = a.H + a.hi, Wp = a.W + a.hi;             // shared-halo grids
  const int Hop = a.Ho + a.ho, Wop = a.Wo + a.ho;
  const int lane = threadIdx.x & 31;
  auto slot = [&](int pix, int c) -> int {
    return SWZ ? (c ^ ((pix * P + (c >> 3)) & 7)) : c;
  };

  for_each_tile(a.b, tiles, [&](long long t) {
    const int band = (int)(t % a.nbands);
    const long long n = t / a.nbands;
    const int p0 = band * a.R, p1 = min(p0 + a.R, a.Ho);
    const int h0 = p0 * a.s, h1 = min((p1 - 1) * a.s + a.k, a.H);
    const int nr = h1 - h0;
    if (a.ho > 0) {
      const int oc16 = a.Cout * ESZ / 16;
      const uint4 z = make_uint4(0, 0, 0, 0);
      uint4 *yb = (uint4 *)a.y;
      if (p1 == a.Ho)                    // bottom halo rows
        for (int v = threadIdx.x; v < a.ho * Wop * oc16; v += blockDim.x)
          yb[((size_t)n * Hop + a.Ho) * Wop * oc16 + v] = z;
      for (int v = threadIdx.x; v < (p1 - p0) * a.ho * oc16; v += blockDim.x) {   // right columns
        const int rr = v / (a.ho * oc16), o = v - rr * a.ho * oc16;
        const size_t rowb = ((size_t)n * Hop + p0 + rr) * Wop * oc16;
        yb[rowb + (size_t)a.Wo * oc16 + o] = z;
      }
    }
    __syncthreads();   // the previous band's pooling is done with smem
    const int npix = nr * a.W;
    const int nv = (npix * P + 31) & ~31;     // warp-uniform trip count
    // the next item's chunks are loaded before the current one is normalised,
    // so every thread keeps two items' global loads in flight
    auto load_item = [&](int v, uint4 (&raw)[CPT]) {
      const int pix = v >> lp, part = v & (P - 1);
      if (pix < npix) {
        int r, col;
        fdivmod(pix, a.W, inv_w, r, col);           // pix < 2^22, W <= 1024: exact
        const char *src = (const char *)a.x +
            ((((size_t)n * Hp + h0 + r) * Wp + col) * C + (size_t)part * CPT * VN) * ESZ;
#pragma unroll
        for (int j = 0; j < CPT; ++j) raw[j] = __ldg((const uint4 *)(src + j * 16));
      } else {
#pragma unroll
        for (int j = 0; j < CPT; ++j) raw[j] = make_uint4(0, 0, 0, 0);
      }
    };
    uint4 nraw[CPT];
    if ((int)threadIdx.x < nv) load_item(threadIdx.x, nraw);
    for (int v = threadIdx.x; v < nv; v += blockDim.x) {
      const int pix = v >> lp, part = v & (P - 1);
      const bool ok = pix < npix;
      Vec16<ST> ch[CPT];
#pragma unroll
      for (int j = 0; j < CPT; ++j) ch[j].from_raw(nraw[j]);
      if (v + (int)blockDim.x < nv) load_item(v + blockDim.x, nraw);
      // window neighbours held by the adjacent lanes of the same pixel
      float tail[HALF], head[HALF];
#pragma unroll
      for (int i = 0; i < HALF; ++i) {
        tail[i] = __shfl_up_sync(0xffffffffu, ch[CPT - 1].v[VN - HALF + i], 1);
        head[i] = __shfl_down_sync(0xffffffffu, ch[0].v[i], 1);
        if (part == 0) tail[i] = 0.f;
        if (part == P - 1 || lane == 31) head[i] = 0.f;
      }
      if (ok) {
        uint8_t *dst = lr_smem + (size_t)pix * chunks * 16;
#pragma unroll
        for (int j = 0; j < CPT; ++j) {
          float sq[VN + 2 * HALF];
#pragma unroll
          for (int q = 0; q < VN + 2 * HALF; ++q) {
            const int o = q - HALF;
            float xv;
            if (o < 0) xv = j > 0 ? ch[j - 1].v[VN + o] : tail[HALF + o];
            else if (o < VN) xv = ch[j].v[o];
            else xv = j + 1 < CPT ? ch[j + 1].v[o - VN] : head[o - VN];
            sq[q] = __fmul_rn(xv, xv);
          }
          Vec16<ST> out;
          lrn_normalise<ST == ST_BF16, 2 * HALF + 1, VN>(sq, ch[j].v, a.lrn_k, a.lrn_alpha_over_n,
                                                         a.lrn_beta, out.v);
          out.store(dst + slot(pix, part * CPT + j) * 16, a.tf32_round);
        }
      }
    }
    __syncthreads();
    // pool (k = s = 1: copy) the normalised rows
    const float inv = 1.f / (float)(a.k * a.k);
    const int ochunks = a.Cout / VN;
    const float inv_oc = 1.f / (float)ochunks;
    const int grp_real = a.ocg / VN, grp_pad = a.ocp / VN;
    const float inv_gp = grp_pad > 0 ? 1.f / (float)grp_pad : 0.f;
    const int nq = a.Wo * ochunks;
    const float inv_nq = 1.f / (float)nq;
    if (ST == ST_BF16 && a.is_max && a.k == 3 && a.s == 2 && (a.Wo - 1) * 2 + 3 <= a.W &&
        (p1 - 1) * 2 + 3 - h0 <= nr) {
      // AlexNet's 3 x 3 / 2 max pool, no window clipped in this band: a thread
      // owns one output column chunk and walks down the band's output rows;
      // the horizontal 3-max of a window's last row is the next window's
      // first (6 instead of 9 smem reads per output; max is exact, so the
      // result is the general path's bit for bit)
      const size_t orow = (size_t)Wop * a.Cout * ESZ;
      for (int v = threadIdx.x; v < nq; v += blockDim.x) {
        int q, oc;
        fdivmod(v, ochunks, inv_oc, q, oc);
        int c = oc;
        bool pad = false;
        if (grp_pad > 0) {
          int gi, j;
          fdivmod(oc, grp_pad, inv_gp, gi, j);
          pad = j >= grp_real;
          c = gi * grp_real + j;
        }
        char *dst = (char *)a.y + ((((size_t)n * Hop + p0) * Wop + q) * a.Cout + oc * VN) * ESZ;
        if (pad) {
          for (int pp = p0; pp < p1; ++pp, dst += orow) *(uint4 *)dst = make_uint4(0, 0, 0, 0);
          continue;
        }
        auto hrow = [&](int r) {                // max over the window's 3 columns of row r
          __nv_bfloat162 m[4];
#pragma unroll
          for (int dc = 0; dc < 3; ++dc) {
            const int pix = r * a.W + 2 * q + dc;
            const uint4 raw = *(const uint4 *)(lr_smem + ((size_t)pix * chunks + slot(pix, c)) * 16);
            const __nv_bfloat162 *h = (const __nv_bfloat162 *)&raw;
#pragma unroll
            for (int j = 0; j < 4; ++j) m[j] = dc ? __hmax2(m[j], h[j]) : h[j];
          }
          return *(const uint4 *)m;
        };
        auto max4 = [](uint4 x, uint4 y) {
          __nv_bfloat162 *a2 = (__nv_bfloat162 *)&x;
          const __nv_bfloat162 *b2 = (const __nv_bfloat162 *)&y;
#pragma unroll
          for (int j = 0; j < 4; ++j) a2[j] = __hmax2(a2[j], b2[j]);
          return x;
        };
        uint4 carry = hrow(p0 * 2 - h0);
        for (int pp = p0; pp < p1; ++pp, dst += orow) {
          const int r0 = pp * 2 - h0;
          const uint4 r2 = hrow(r0 + 2);
          *(uint4 *)dst = max4(max4(carry, hrow(r0 + 1)), r2);
          carry = r2;
        }
      }
      return;
    }
    for (int v = threadIdx.x; v < (p1 - p0) * nq; v += blockDim.x) {
      int rr, q, oc;
      if (nq <= 1024) fdivmod(v, nq, inv_nq, rr, q);   // fdivmod's exact range
      else { rr = v / nq; q = v - rr * nq; }
      fdivmod(q, ochunks, inv_oc, q, oc);
      const int pp = p0 + rr;
      int c = oc;
      bool pad = false;
      if (grp_pad > 0) {
        int gi, j;
        fdivmod(oc, grp_pad, inv_gp, gi, j);
        pad = j >= grp_real;
        c = gi * grp_real + j;
      }
      char *dst = (char *)a.y + ((((size_t)n * Hop + pp) * Wop + q) * a.Cout + oc * VN) * ESZ;
      const int rs = pp * a.s - h0, re = min(rs + a.k, nr);
      const int cs = q * a.s, ce = min(cs + a.k, a.W);
      if (ST == ST_BF16 && a.is_max) {
        __nv_bfloat162 m[4];
        const __nv_bfloat162 ninf = __float2bfloat162_rn(-INFINITY);
        const __nv_bfloat162 zero = __float2bfloat162_rn(0.f);
#pragma unroll
        for (int j = 0; j < 4; ++j) m[j] = pad ? zero : ninf;
        auto take = [&](int pix) {
          const uint4 raw = *(const uint4 *)(lr_smem + ((size_t)pix * chunks + slot(pix, c)) * 16);
          const __nv_bfloat162 *h = (const __nv_bfloat162 *)&raw;
#pragma unroll
          for (int j = 0; j < 4; ++j) m[j] = __hmax2(m[j], h[j]);
        };
        if (!pad) {
          if (re - rs == 3 && ce - cs == 3) {      // AlexNet's 3 x 3 windows, unclipped
            const int pix0 = rs * a.W + cs;
#pragma unroll
            for (int dr = 0; dr < 3; ++dr)
#pragma unroll
              for (int dc = 0; dc < 3; ++dc) take(pix0 + dr * a.W + dc);
          } else {
            for (int r = rs; r < re; ++r)
              for (int col = cs; col < ce; ++col) take(r * a.W + col);
          }
        }
        *(uint4 *)dst = *(const uint4 *)m;
        continue;
      }
      Vec16<ST> acc, cur;
#pragma unroll
      for (int j = 0; j < VN; ++j) acc.v[j] = pad ? 0.f : (a.is_max ? -INFINITY : 0.f);
      if (!pad) {
        for (int r = rs; r < re; ++r)
          for (int col = cs; col < ce; ++col) {
            const int pix = r * a.W + col;
            cur.load(lr_smem + ((size_t)pix * chunks + slot(pix, c)) * 16);
#pragma unroll
            for (int j = 0; j < VN; ++j)
              acc.v[j] = a.is_max ? fmaxf(acc.v[j], cur.v[j]) : acc.v[j] + cur.v[j];
          }
        if (!a.is_max)
#pragma unroll
          for (int j = 0; j < VN; ++j) acc.v[j] *= inv;
      }
      acc.store(dst, a.is_max ? 0 : a.tf32_round);
    }
  });
}

// chunks per lane of lrn_reg_kernel for C stored channels (0 = not supported):
// 8 (swizzled) when the chunk count is a multiple of 8, else 6 or 3 with a
// power-of-two lane count per pixel.
static int lrn_reg_cpt(int st, int C) {
  const int vn = st == ST_BF16 ? 8 : 4;
  if (C % vn) return 0;
  const int chunks = C / vn;
  auto pow2_le32 = [](int p) { return p >= 1 && p <= 32 && (p & (p - 1)) == 0; };
  const char *e = exp_env("PCNN_LRN_CPT");        // tuning experiments
  const int want = e ? atoi(e) : 0;
  if (want == 3 && chunks % 3 == 0 && pow2_le32(chunks / 3)) return 3;
  if (chunks % 8 == 0 && pow2_le32(chunks / 8)) return 8;
  if (chunks % 6 == 0 && pow2_le32(chunks / 6)) return 6;
  if (chunks % 3 == 0 && pow2_le32(chunks / 3)) return 3;
  return 0;
}

constexpr int LB_SMEM_BUDGET = 100 * 1024;

// output rows per band so that the band's staged rows fit LB_SMEM_BUDGET
static bool use_lrn_reg(int st, int C, int lrn, int W) {
  if (W > 1024) return false;                    // fdivmod's exact range (pixel -> row, col)
  const char *e = exp_env("PCNN_LRN_BAND");     // A/B tests: the staged band kernel
  const bool off = e && e[0] == '1';
  return lrn == 5 && !off && lrn_reg_cpt(st, C) > 0;
}

// Small batches: fewer rows per band until the launch has ~2 CTAs per SM (the
// bands overlap by k - s input rows, recomputed; results do not depend on R).
static int lrn_band_rows(int st, int B, int W, int C, int k, int s, int Ho, int lrn) {
  const int esz = st == ST_BF16 ? 2 : 4;
  const size_t row = (size_t)W * (C * esz + (use_lrn_reg(st, C, lrn, W) ? 0 : 16));
  const char *e = exp_env("PCNN_LB_KB");          // tuning experiments
  const size_t budget = e ? (size_t)atoi(e) * 1024 : (size_t)LB_SMEM_BUDGET;
  int R = 1;
  while (R < Ho && (size_t)((R) * s + k) * row <= budget) ++R;
  while (R > 1 && (long long)B * ((Ho + R - 1) / R) < kBandTargetCtas) --R;
  return R;
}

constexpr int LP_SMEM_BUDGET = 48 * 1024;

// Output columns per tile so that the staged rows fit the smem budget.
static int lrn_pool_cols(int st, int W, int C, int lrn, int k, int s, int Wo) {
  const int esz = st == ST_BF16 ? 2 : 4;
  const size_t per_col = (size_t)k * C * esz * (lrn ? 2 : 1);
  int Q = Wo;
  while (Q > 1 && (size_t)((Q - 1) * s + k) * per_col > LP_SMEM_BUDGET) Q = (Q + 1) / 2;
  (void)W;
  return Q;
}

int lrn_pool_occupancy(int st) {
  int n = 0;
  if (st == ST_BF16)
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n, lrn_pool_kernel<ST_BF16, 5>, 256, LP_SMEM_BUDGET);
  else
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n, lrn_pool_kernel<ST_F32, 5>, 256, LP_SMEM_BUDGET);
  return n > 0 ? n : 1;
}

template <int ST, int LS>
static cudaError_t lrn_pool_launch(const LrnPoolArgs &a, int grid, size_t smem, cudaStream_t s) {
  if (smem > 48 * 1024)
    cudaFuncSetAttribute(lrn_pool_kernel<ST, LS>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                         (int)smem);
  launch_pdl(lrn_pool_kernel<ST, LS>, dim3(grid), dim3(256), smem, s, a);
  return cudaGetLastError();
}

template <int ST>
static cudaError_t lrn_pool_dispatch(const LrnPoolArgs &a, int grid, size_t smem, cudaStream_t s) {
  switch (a.lrn_size) {
    case 0: return lrn_pool_launch<ST, 0>(a, grid, smem, s);
    case 1: return lrn_pool_launch<ST, 1>(a, grid, smem, s);
    case 3: return lrn_pool_launch<ST, 3>(a, grid, smem, s);
    case 5: return lrn_pool_launch<ST, 5>(a, grid, smem, s);
    case 7: return lrn_pool_launch<ST, 7>(a, grid, smem, s);
    case 9: return lrn_pool_launch<ST, 9>(a, grid, smem, s);
  }
  return cudaErrorInvalidValue;
}

long long lrn_pool_tiles(int st, int B, int W, int C, int lrn, int k, int s, int Ho, int Wo) {
  if (lrn) {
    const int R = lrn_band_rows(st, B, W, C, k, s, Ho, lrn);
    return (long long)B * ((Ho + R - 1) / R);
  }
  const int Q = lrn_pool_cols(st, W, C, lrn, k, s, Wo);
  return (long long)B * Ho * ((Wo + Q - 1) / Q);
}


// Plain pooling (no LRN, no group padding) straight from global memory: one
// thread per (output pixel, 16 B channel chunk), chunk fastest, so each warp
// reads whole runs of input pixels; K = 2 / 3 windows are unrolled (VGG 2x2
// s2, AlexNet 3x3 s2), overlapping windows re-hit L1.  Writes the output
// halo zeros.  Same max / mean arithmetic as lrn_pool_kernel.
template <int ST, int K>
__global__ void __launch_bounds__(256)
pool_direct_kernel(const uint4 *__restrict__ x, uint4 *__restrict__ y, int B, int H, int W,
                   int chunks, int kk, int s, int is_max, int Ho, int Wo, int hi, int ho,
                   int tf32_round, int ochunks, int grp_real, int grp_pad, Budget bud) {
  pdl_enter();   // PDL: wait for the previous kernel, let the next one launch
  constexpr int VN = Vec16<ST>::N;
  const int k = K > 0 ? K : kk;
  const int Hp = H + hi, Wp = W + hi, Hop = Ho + ho, Wop = Wo + ho;   // shared-halo grids
  // output chunks: `chunks` input chunks, or (grp_pad > 0) each group's
  // grp_real chunks padded with zeros to grp_pad (the layout a grouped conv
  // reads with whole 128-B TMA slabs)
  const long long total = (long long)B * Hop * Wop * ochunks;
  const float inv = 1.f / (float)(k * k);
  if (threadIdx.x == 0) census_mark(bud);
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < total;
       i += (long long)gridDim.x * blockDim.x) {
    int ch = (int)(i % ochunks);
    const long long pix = i / ochunks;
    const int q = (int)(pix % Wop);
    const long long t = pix / Wop;
    const int p = (int)(t % Hop);
    const long long n = t / Hop;
    bool pad = false;
    if (grp_pad > 0) {
      const int gi = ch / grp_pad, j = ch - gi * grp_pad;
      pad = j >= grp_real;
      ch = gi * grp_real + j;
    }
    if (pad || p < 0 || p >= Ho || q < 0 || q >= Wo) {
      y[i] = make_uint4(0, 0, 0, 0);
      continue;
    }
    const int r0 = p * s, c0 = q * s;
    const int re = min(r0 + k, H), ce = min(c0 + k, W);
    const uint4 *base = x + (((size_t)n * Hp + r0) * Wp + c0) * chunks + ch;
    if (ST == ST_BF16 && is_max) {
      __nv_bfloat162 m[4];
      const __nv_bfloat162 ninf = __float2bfloat162_rn(-INFINITY);
#pragma unroll
      for (int j = 0; j < 4; ++j) m[j] = ninf;
      auto take = [&](const uint4 *ptr) {
        const uint4 raw = __ldg(ptr);
        const __nv_bfloat162 *h2 = (const __nv_bfloat162 *)&raw;
#pragma unroll
        for (int j = 0; j < 4; ++j) m[j] = __hmax2(m[j], h2[j]);
      };
      if (K > 0 && re - r0 == K && ce - c0 == K) {
#pragma unroll
        for (int dr = 0; dr < (K > 0 ? K : 1); ++dr)
#pragma unroll
          for (int dc = 0; dc < (K > 0 ? K : 1); ++dc) take(base + ((size_t)dr * Wp + dc) * chunks);
      } else {
        for (int r = r0; r < re; ++r)
          for (int c = c0; c < ce; ++c) take(base + ((size_t)(r - r0) * Wp + (c - c0)) * chunks);
      }
      y[i] = *(const uint4 *)m;
      continue;
    }
    Vec16<ST> acc, cur;
#pragma unroll
    for (int j = 0; j < VN; ++j) acc.v[j] = is_max ? -INFINITY : 0.f;
    for (int r = r0; r < re; ++r)
      for (int c = c0; c < ce; ++c) {
        cur.from_raw(__ldg(base + ((size_t)(r - r0) * Wp + (c - c0)) * chunks));
#pragma unroll
        for (int j = 0; j < VN; ++j)
          acc.v[j] = is_max ? fmaxf(acc.v[j], cur.v[j]) : acc.v[j] + cur.v[j];
      }
    if (!is_max)
#pragma unroll
      for (int j = 0; j < VN; ++j) acc.v[j] *= inv;
    acc.store(y + i, is_max ? 0 : tf32_round);
  }
}

cudaError_t launch_lrn_pool(const void *x, void *y, int st, int tf32_round, int B, int H, int W,
                            int C, int lrn_size, float alpha, float beta, float kk, int k,
                            int s, int is_max, int Ho, int Wo, int out_groups, int out_cg_pad,
                            int in_halo, int out_halo, const Budget &b, int grid,
                            cudaStream_t stream) {
  const int vn = st == ST_BF16 ? 8 : 4;
  if (C % vn) return cudaErrorInvalidValue;
  const int ocg = out_groups > 0 ? C / out_groups : 0;
  const int ocp = out_groups > 0 ? out_cg_pad : 0;
  if (out_groups > 0 && (C % out_groups || ocg % vn || ocp % vn || ocp < ocg))
    return cudaErrorInvalidValue;
  if (lrn_size == 0 && !b.gated && !exp_env("PCNN_OLD_POOL")) {
    const int chunks = C / vn;
    const int gr = out_groups > 0 ? ocg / vn : 0, gp = out_groups > 0 ? ocp / vn : 0;
    const int ochunks = out_groups > 0 ? out_groups * gp : chunks;
    const long long total = (long long)B * (Ho + out_halo) * (Wo + out_halo) * ochunks;
    const int g = (int)std::min<long long>((total + 255) / 256, 148LL * 16);
#define PCNN_PD(STT, KK)                                                                       \
  launch_pdl(pool_direct_kernel<STT, KK>, dim3(g), dim3(256), 0, stream, (const uint4 *)x, (uint4 *)y, B, H, W,    \
                                                     chunks, k, s, is_max, Ho, Wo, in_halo,    \
                                                     out_halo, tf32_round, ochunks, gr, gp, b)
    if (st == ST_BF16) {
      if (k == 2) PCNN_PD(ST_BF16, 2); else if (k == 3) PCNN_PD(ST_BF16, 3); else PCNN_PD(ST_BF16, 0);
    } else {
      if (k == 2) PCNN_PD(ST_F32, 2); else if (k == 3) PCNN_PD(ST_F32, 3); else PCNN_PD(ST_F32, 0);
    }
#undef PCNN_PD
    return cudaGetLastError();
  }
  LrnPoolArgs a;
  a.x = x;
  a.y = y;
  a.B = B;
  a.H = H;
  a.W = W;
  a.C = C;
  a.lrn_size = lrn_size;
  a.lrn_alpha_over_n = lrn_size > 0 ? alpha / (float)lrn_size : 0.f;
  a.lrn_beta = beta;
  a.lrn_k = kk;
  a.k = k;
  a.s = s;
  a.is_max = is_max;
  a.Ho = Ho;
  a.Wo = Wo;
  a.Q = lrn_pool_cols(st, W, C, lrn_size > 0, k, s, Wo);
  a.nqt = (Wo + a.Q - 1) / a.Q;
  a.tf32_round = tf32_round;
  a.ocg = ocg;
  a.ocp = ocp;
  a.Cout = out_groups > 0 ? out_groups * ocp : C;
  a.hi = in_halo;
  a.ho = out_halo;
  a.b = b;
  const int esz = st == ST_BF16 ? 2 : 4;
  if (use_lrn_reg(st, C, lrn_size, W)) {
    a.R = lrn_band_rows(st, B, W, C, k, s, Ho, lrn_size);
    a.nbands = (Ho + a.R - 1) / a.R;
    const size_t smem = (size_t)(min((a.R - 1) * s + k, H)) * W * C * esz;
    if (smem > 200 * 1024) return cudaErrorInvalidValue;
    const int cpt = lrn_reg_cpt(st, C);
    static const bool occ3 = [] {                 // experiment: 3 CTAs / SM (<= 85 regs)
      const char *e = exp_env("PCNN_LRN_OCC3");
      return e && e[0] == '1';
    }();
#define PCNN_LR(STT, CP)                                                                        \
  do {                                                                                          \
    if (occ3) {                                                                                 \
      if (smem > 48 * 1024)                                                                     \
        cudaFuncSetAttribute(lrn_reg_kernel<STT, CP, 3>,                                        \
                             cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);           \
      launch_pdl(lrn_reg_kernel<STT, CP, 3>, dim3(grid), dim3(256), smem, stream, a);                               \
    } else {                                                                                    \
      if (smem > 48 * 1024)                                                                     \
        cudaFuncSetAttribute(lrn_reg_kernel<STT, CP>,                                           \
                             cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);           \
      launch_pdl(lrn_reg_kernel<STT, CP>, dim3(grid), dim3(256), smem, stream, a);                                  \
    }                                                                                           \
  } while (0)
    if (st == ST_BF16) {
      if (cpt == 8) PCNN_LR(ST_BF16, 8); else if (cpt == 6) PCNN_LR(ST_BF16, 6); else PCNN_LR(ST_BF16, 3);
    } else {
      if (cpt == 8) PCNN_LR(ST_F32, 8); else if (cpt == 6) PCNN_LR(ST_F32, 6); else PCNN_LR(ST_F32, 3);
    }
#undef PCNN_LR
    return cudaGetLastError();
  }
  if (lrn_size > 0 && (lrn_size == 5 || lrn_size == 3)) {
    // band kernel (every LRN, fused with a following pool or not)
    a.R = lrn_band_rows(st, B, W, C, k, s, Ho, lrn_size);
    a.nbands = (Ho + a.R - 1) / a.R;
    const size_t smem = (size_t)(min((a.R - 1) * s + k, H)) * W * (C * esz + 16);
    if (smem > 200 * 1024) return cudaErrorInvalidValue;
#define PCNN_LB(STT, LSS)                                                                       \
  do {                                                                                          \
    if (smem > 48 * 1024)                                                                       \
      cudaFuncSetAttribute(lrn_band_kernel<STT, LSS>,                                           \
                           cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);             \
    launch_pdl(lrn_band_kernel<STT, LSS>, dim3(grid), dim3(256), smem, stream, a);                                  \
  } while (0)
    if (st == ST_BF16) {
      if (lrn_size == 5) PCNN_LB(ST_BF16, 5); else PCNN_LB(ST_BF16, 3);
    } else {
      if (lrn_size == 5) PCNN_LB(ST_F32, 5); else PCNN_LB(ST_F32, 3);
    }
#undef PCNN_LB
    return cudaGetLastError();
  }
  const size_t smem = (size_t)k * ((a.Q - 1) * s + k) * C * esz * (lrn_size > 0 ? 2 : 1);
  if (smem > 200 * 1024) return cudaErrorInvalidValue;
  if (st == ST_BF16) return lrn_pool_dispatch<ST_BF16>(a, grid, smem, stream);
  if (lrn_size > 9) return cudaErrorInvalidValue;   // fp32 chunk holds 4 channels
  return lrn_pool_dispatch<ST_F32>(a, grid, smem, stream);
}

// ------------------------------------------------------------ NEXT-1: interpolation
// Perforation-interpolation (Fig. 11, reading R13): every output pixel
// of the layer takes the channel vector of its nearest kept grid position
// (kept rows 0, sh, 2sh, ...; ties to the lower one).  A pure copy: one thread
// per (output pixel, 16 B chunk), chunk fastest so loads and stores coalesce.
__device__ __forceinline__ int perf_src(int p, int s, int n) {
  const int lo = p / s * s, hi = lo + s;
  return (hi < n && hi - p < p - lo) ? hi / s : lo / s;
}

__global__ void __launch_bounds__(256)
perf_interp_kernel(const uint4 *__restrict__ t, uint4 *__restrict__ y, int B, int Ho, int Wo,
                   int sh, int sw, int chunks, int ho) {
  pdl_enter();   // PDL: wait for the previous kernel, let the next one launch
  const int Hk = (Ho + sh - 1) / sh, Wk = (Wo + sw - 1) / sw;
  const int Hp = Ho + ho, Wp = Wo + ho;               // shared-halo output grid
  const long long total = (long long)B * Hp * Wp * chunks;
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < total;
       i += (long long)gridDim.x * blockDim.x) {
    const int ch = (int)(i % chunks);
    const long long pix = i / chunks;
    const int q = (int)(pix % Wp);
    const long long r = pix / Wp;
    const int p = (int)(r % Hp);
    const long long n = r / Hp;
    uint4 v = make_uint4(0, 0, 0, 0);
    if (p >= 0 && p < Ho && q >= 0 && q < Wo) {
      const long long src = ((n * Hk + perf_src(p, sh, Ho)) * Wk + perf_src(q, sw, Wo)) * chunks + ch;
      v = __ldg(t + src);
    }
    y[i] = v;
  }
}

cudaError_t launch_perf_interp(const void *t, void *y, int st, int B, int Ho, int Wo, int sh,
                               int sw, int Cs, int ho, cudaStream_t s) {
  const int esz = st == ST_BF16 ? 2 : 4;
  if ((Cs * esz) % 16) return cudaErrorInvalidValue;
  const int chunks = Cs * esz / 16;
  const long long total = (long long)B * (Ho + ho) * (Wo + ho) * chunks;
  const int grid = (int)std::min<long long>((total + 255) / 256, 148LL * 16);
  launch_pdl(perf_interp_kernel, dim3(grid), dim3(256), 0, s, (const uint4 *)t, (uint4 *)y, B, Ho, Wo, sh, sw,
                                          chunks, ho);
  return cudaGetLastError();
}

// ------------------------------------------------------------ a7: softmax + entropy
// One warp per image: max and sum by warp shuffles (eq. 2).
// H = ln S - sum_j p_j (z_j - max), algebraically -sum p ln p (reading R6).
// NR > 0: the row (N <= 32 * NR) is held in registers, read once; NR = 0:
// generic strided loops.  Same per-element arithmetic either way.
template <int NR>
__global__ void softmax_entropy_kernel(const float *__restrict__ z, float *p,
                                       float *h, int B, int N) {
  pdl_enter();   // PDL: wait for the previous kernel, let the next one launch
  const int warp = (blockIdx.x * blockDim.x + threadIdx.x) / 32;
  const int lane = threadIdx.x % 32;
  if (warp >= B) return;
  const float *zr = z + (size_t)warp * N;
  float m = -INFINITY;
  float v[NR > 0 ? NR : 1];
  if constexpr (NR > 0) {
#pragma unroll
    for (int i = 0; i < NR; ++i) {
      const int j = lane + 32 * i;
      v[i] = j < N ? __ldg(zr + j) : -INFINITY;
      m = fmaxf(m, v[i]);
    }
  } else {
    for (int j = lane; j < N; j += 32) m = fmaxf(m, zr[j]);
  }
  for (int o = 16; o; o >>= 1) m = fmaxf(m, __shfl_xor_sync(0xffffffffu, m, o));
  float s = 0.f, sz = 0.f;
  if constexpr (NR > 0) {
#pragma unroll
    for (int i = 0; i < NR; ++i) {
      if (lane + 32 * i < N) {
        const float d = v[i] - m;
        const float e = expf(d);
        s += e;
        sz += e * d;
        v[i] = e;
      }
    }
  } else {
    for (int j = lane; j < N; j += 32) {
      const float d = zr[j] - m;
      const float e = expf(d);
      s += e;
      sz += e * d;
    }
  }
  for (int o = 16; o; o >>= 1) {
    s += __shfl_xor_sync(0xffffffffu, s, o);
    sz += __shfl_xor_sync(0xffffffffu, sz, o);
  }
  const float inv = 1.f / s;
  if (p) {
    if constexpr (NR > 0) {
#pragma unroll
      for (int i = 0; i < NR; ++i)
        if (lane + 32 * i < N) p[(size_t)warp * N + lane + 32 * i] = v[i] * inv;
    } else {
      for (int j = lane; j < N; j += 32) p[(size_t)warp * N + j] = expf(zr[j] - m) * inv;
    }
  }
  if (h && lane == 0) h[warp] = logf(s) - sz * inv;
}
cudaError_t launch_softmax_entropy(const float *z, float *p, float *h, int B,
                                   int N, cudaStream_t s) {
  // two warps (images) per CTA: a 256-image batch spreads over 128 SMs
  const int warps_per_block = 2;
  const int grid = (B + warps_per_block - 1) / warps_per_block;
  if (N <= 32 * 32)
    launch_pdl(softmax_entropy_kernel<32>, dim3(grid), dim3(warps_per_block * 32), 0, s, z, p, h, B, N);
  else
    launch_pdl(softmax_entropy_kernel<0>, dim3(grid), dim3(warps_per_block * 32), 0, s, z, p, h, B, N);
  return cudaGetLastError();
}

}  // namespace pcnn
