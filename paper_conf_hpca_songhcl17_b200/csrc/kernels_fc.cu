// kernels_fc.cu -- weight-streaming tcgen05 FC layer for sm_100a (a6; K2).
//
// What it computes ("classifier layers"; R5):
//   Y[b][n] = act( sum_k W[n][k] X[b][k] + bias[n] )   for every image b.
// AlexNet / VGG-16 FC layers hold 96% / 89% of the weights; at batch
// <= ~260 (BF16) their arithmetic intensity is below the ridge, so the layer
// is a weight stream that every SM must help pull.
//
// Mapping ("swap AB", CTA pair): the UMMA M dimension is 256 weight rows per
// CTA pair (cta_group::2; 128 rows in each CTA's shared memory), the UMMA N
// dimension is the batch (nb = 16..256 images of a chunk; each CTA of the pair
// loads nb / 2 of them), K is the input feature.  Per K-block a CTA therefore
// ingests 16 KB of weights + nb x 64 B of activations for a 128 x nb x 64
// share of the MMA -- the pair halves the activation bytes each SM must pull
// through L2 (the measured bound of this layer at large batch: ~40 B/clk/SM).
// Weights are pre-tiled on the host into contiguous 16 KB tiles
// ([row block][K-block][128 rows][128 B]), so each TMA box is one run of HBM.
// The accumulator lanes are weight rows: one image's outputs leave as
// coalesced stores along n.
//
// K split (deterministic, batch-independent): `splits` CTA pairs share one
// (256-row block, batch chunk) unit; pair j accumulates K-blocks
// [j*KB/s, (j+1)*KB/s) and writes its FP32 partial tile to the workspace
// (L2-resident).  The 2*splits CTAs of the unit meet at a counter in global
// memory (release / acquire at GPU scope; all CTAs of the launch are
// co-resident: grid <= SMs, one CTA per SM by shared memory), then CTA i of
// them sums rows [i*256/(2s), (i+1)*256/(2s)) over the s partials in split
// order 0..s-1, adds bias, applies ReLU and rounds to the storage precision.
// The split count and K ranges depend only on (N, K, SM count), never on the
// batch or the SM budget, and every image is its own UMMA column, so an
// image's logits are bitwise identical for any batch size, chunking or budget.
//
// PDL: the weights do not depend on the previous layer, so the producer
// streams the first ring of weight tiles before griddepcontrol.wait.
//
// CTA = 10 warps: warp 0 TMA producer, warp 1 TMEM allocator + MMA issuer
// (leader CTA), warps 2..9 epilogue / reduction (TMEM lane quarter = warp % 4,
// two warps per quarter taking alternate 32-column chunks).
#include <algorithm>

#include "budget.cuh"
#include "pcnn_internal.h"
#include "tc_ptx.cuh"

namespace pcnn {

constexpr int FC_THREADS = 320;        // producer, MMA, 8 epilogue / reduction warps
constexpr int FC_EPI = FC_THREADS - 64; // epilogue threads
constexpr int FC_STAGE_BUDGET = 200 * 1024;
constexpr int FC_MAX_STAGES = 16;
constexpr int FC_W_TILE = 128 * 128;          // one weight tile: 128 rows x 128 B
constexpr int FC_SM_BAR = FC_STAGE_BUDGET;
constexpr int FC_SM_FULL = FC_SM_BAR;
constexpr int FC_SM_EMPTY = FC_SM_FULL + 8 * FC_MAX_STAGES;
constexpr int FC_SM_TFULL = FC_SM_EMPTY + 8 * FC_MAX_STAGES;
constexpr int FC_SM_TEMPTY = FC_SM_TFULL + 8;
constexpr int FC_SM_TMEMPTR = FC_SM_TEMPTY + 8;
constexpr int FC_SM_TOTAL = FC_SM_TMEMPTR + 16;
constexpr size_t FC_SMEM_BYTES = FC_SM_TOTAL + 1024;
constexpr int FC_ROWS = 256;                  // weight rows per CTA pair (UMMA M)

#ifndef PCNN_TC_PROF
#define PCNN_TC_PROF 0
#endif
// Debug timeline (prof build, PCNN_TC_PROFILE=1; globaltimer ns summed over
// CTAs, from each CTA's PDL wait): 0 entry -> wait, 1 accumulator ready,
// 2 partial stored, 3 split-K peers met, 4 reduction done, 5 exit, 6 CTAs,
// 7 ~min entry, 8 max exit, 9 ~min wait
__device__ unsigned long long g_fc_prof[16];
__device__ __forceinline__ unsigned long long fc_gtimer() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}

struct FcArgs {
  int prof;
  int N, B;              // output features (weight rows), batch rows of X
  int kblocks, kbps;     // K-blocks of Kpad, K-blocks per split
  int splits;            // CTA pairs per unit (K split)
  int nb;                // UMMA N (batch columns per chunk)
  int rblocks, chunks, units, groups;
  int stages, stage_bytes, tmem_cols;
  int kbe;               // K elements per K-block (128 B)
  int relu, out_mode, ldy;
  void *y;
  float *ws;             // [splits][B][N] fp32 partials (splits > 1)
  unsigned *sem;         // [2][units] arrival / departure counters (zero between launches)
  const float *bias;
  Budget b;
};

template <int ST>
__device__ __forceinline__ uint32_t fc_idesc(int nb) {
  const uint32_t fmt = ST == ST_BF16 ? 1u : 2u;
  return (1u << 4) | (fmt << 7) | (fmt << 10) | ((uint32_t)(nb >> 3) << 17) |
         ((uint32_t)(FC_ROWS >> 4) << 24);
}

__device__ __forceinline__ float fc_act(float v, int relu) { return relu ? fmaxf(v, 0.f) : v; }

__device__ __forceinline__ void fc_store(void *y, size_t idx, float v, int out_mode) {
  if (out_mode == OUT_BF16) {
    ((__nv_bfloat16 *)y)[idx] = __float2bfloat16_rn(v);
  } else {
    if (out_mode == OUT_F32_TF32) {
      unsigned r;
      asm("cvt.rna.tf32.f32 %0, %1;" : "=r"(r) : "f"(v));
      v = __uint_as_float(r);
    }
    ((float *)y)[idx] = v;
  }
}

__device__ __forceinline__ void epi_bar() {          // the 8 epilogue warps only
  asm volatile("bar.sync 1, %0;" ::"n"(FC_EPI) : "memory");
}
__device__ __forceinline__ unsigned ld_acquire(const unsigned *p) {
  unsigned v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}

// Split-K reduction of one unit by CTA `idx` (0 .. 2s-1) of the unit: rows
// [idx * 256 / (2s), ...) for every image of the chunk, each output the sum of
// the s partials in split order 0..s-1 (+ bias, activation, rounding).  Four
// consecutive rows per thread (16-B loads); the partials of 8 / s images are
// all in flight before the first add (the loads are L2-latency bound).
template <int S>
__device__ __forceinline__ void fc_reduce(const FcArgs &a, int rb, int ch, int idx, int t) {
  constexpr int s = S, rows = FC_ROWS / (2 * S);
  constexpr int IMG = S >= 8 ? 1 : 8 / S;
  const int b0 = ch * a.nb, ncols = min(a.nb, a.B - b0);
  const size_t sBN = (size_t)a.B * a.N;
  const int nbase = rb * FC_ROWS + idx * rows;
  if ((a.N & 3) == 0) {
    constexpr int r4 = rows / 4, bstep = FC_EPI / r4;
    const int q = t % r4, bsub = t / r4;
    const int n = nbase + 4 * q;
    if (bsub >= bstep || n >= a.N) return;
    const float4 bias = *(const float4 *)(a.bias + n);
    for (int bi0 = bsub; bi0 < ncols; bi0 += IMG * bstep) {
      float4 v[IMG][S];
#pragma unroll
      for (int h = 0; h < IMG; ++h) {
        const int bi = bi0 + h * bstep;
        if (bi < ncols) {
          const size_t o = (size_t)(b0 + bi) * a.N + n;
#pragma unroll
          for (int j = 0; j < S; ++j)
            v[h][j] = __ldcg((const float4 *)(a.ws + (size_t)j * sBN + o));   // L2: peers' writes
        }
      }
#pragma unroll
      for (int h = 0; h < IMG; ++h) {
        const int bi = bi0 + h * bstep;
        if (bi >= ncols) break;
        float4 acc = v[h][0];
#pragma unroll
        for (int j = 1; j < S; ++j) {
          acc.x += v[h][j].x;
          acc.y += v[h][j].y;
          acc.z += v[h][j].z;
          acc.w += v[h][j].w;
        }
        const size_t yo = (size_t)(b0 + bi) * a.ldy + n;
        fc_store(a.y, yo, fc_act(acc.x + bias.x, a.relu), a.out_mode);
        fc_store(a.y, yo + 1, fc_act(acc.y + bias.y, a.relu), a.out_mode);
        fc_store(a.y, yo + 2, fc_act(acc.z + bias.z, a.relu), a.out_mode);
        fc_store(a.y, yo + 3, fc_act(acc.w + bias.w, a.relu), a.out_mode);
      }
    }
    return;
  }
  for (int e = t; e < rows * ncols; e += FC_EPI) {       // general N: one output per step
    const int r = e % rows, bi = e / rows;
    const int n = nbase + r;
    if (n >= a.N) continue;
    const size_t off = (size_t)(b0 + bi) * a.N + n;
    float v[S];
#pragma unroll
    for (int j = 0; j < S; ++j) v[j] = __ldcg(a.ws + (size_t)j * sBN + off);
    float acc = v[0];
#pragma unroll
    for (int j = 1; j < S; ++j) acc += v[j];
    fc_store(a.y, (size_t)(b0 + bi) * a.ldy + n, fc_act(acc + __ldg(&a.bias[n]), a.relu),
             a.out_mode);
  }
}

template <int ST>
__global__ void __launch_bounds__(FC_THREADS, 1)
fc_tc_kernel(const __grid_constant__ CUtensorMap tmap_w, const __grid_constant__ CUtensorMap tmap_x,
             const FcArgs a) {
  extern __shared__ uint8_t smem_raw[];
  const bool prof = PCNN_TC_PROF && a.prof;
  const unsigned long long t_entry = prof ? fc_gtimer() : 0;
  unsigned long long t_full = 0, t_st = 0, t_met = 0, t_red = 0;
  uint8_t *smem = (uint8_t *)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
  const uint32_t sbase = smem_u32(smem);
  const int tid = threadIdx.x;
  const int warp = __shfl_sync(0xffffffffu, tid >> 5, 0), lane = tid & 31;
  const uint32_t rank = cluster_ctarank();                 // 0 = leader of the pair
  const int s = a.splits;
  const int pair = blockIdx.x >> 1;
  const int split = pair % s, grp = pair / s;              // K split, unit group
  const int stages = a.stages;
  const uint32_t sbytes = (uint32_t)a.stage_bytes;

  if (tid == 0) {
    for (int i = 0; i < stages; ++i) {
      mbar_init(sbase + FC_SM_FULL + 8 * i, 1);
      mbar_init(sbase + FC_SM_EMPTY + 8 * i, 1);
    }
    mbar_init(sbase + FC_SM_TFULL, 1);
    mbar_init(sbase + FC_SM_TEMPTY, 2 * (FC_EPI / 32));     // epilogue warps of both CTAs
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    census_mark(a.b);
  }
  if (warp == 1) {
    asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(
                     sbase + FC_SM_TMEMPTR),
                 "r"(a.tmem_cols));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;");
  }
  tc_fence_before();
  cluster_sync();
  tc_fence_after();
  const uint32_t tmem_base = *(volatile uint32_t *)(smem + FC_SM_TMEMPTR);

  // balanced, never-empty K ranges: split j takes [j KB / s, (j + 1) KB / s)
  const int k0 = (int)((long long)split * a.kblocks / s);
  const int k1 = (int)((long long)(split + 1) * a.kblocks / s);
  // PDL prefetch: the first unit's first ring of weight tiles (the full
  // barrier's byte count -- on the leader -- covers the activation halves
  // loaded after the wait)
  int pre = 0;
  if (warp == 0 && lane == 0 && grp < a.units) {
    asm volatile("prefetch.tensormap [%0];" ::"l"((uint64_t)&tmap_w) : "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"((uint64_t)&tmap_x) : "memory");
    const int rb0 = grp / a.chunks;
    pre = min(stages, k1 - k0);
    for (int i = 0; i < pre; ++i) {
      const uint32_t fb = sbase + FC_SM_FULL + 8 * i;
      if (rank == 0) mbar_arrive_expect_tx(fb, 2 * sbytes);
      tma_load_4d<2>(sbase + i * sbytes, &tmap_w, fb, 0, 0, k0 + i, rb0 * 2 + (int)rank);
    }
  }
  pdl_enter();
  const unsigned long long t_wait = prof ? fc_gtimer() : 0;

  uint32_t stage = 0, phase = 0;
  int lt = 0;
  for (int u = grp; u < a.units; u += a.groups, ++lt) {
    // row-block-major: concurrently running groups share one weight slice
    const int rb = u / a.chunks, ch = u - rb * a.chunks;
    if (warp == 0) {
      // ------------------------------------------------ TMA producer (both CTAs)
      if (lane == 0) {
        for (int kb = k0; kb < k1; ++kb) {
          const uint32_t fb = sbase + FC_SM_FULL + 8 * stage;
          const uint32_t dst = sbase + stage * sbytes;
          if (lt > 0 || kb - k0 >= pre) {        // not prefetched before the PDL wait
            mbar_wait(sbase + FC_SM_EMPTY + 8 * stage, phase ^ 1);
            if (rank == 0) mbar_arrive_expect_tx(fb, 2 * sbytes);
            tma_load_4d<2>(dst, &tmap_w, fb, 0, 0, kb, rb * 2 + (int)rank);
          }
          tma_load_2d_2sm(dst + FC_W_TILE, &tmap_x, fb, kb * a.kbe,
                          ch * a.nb + (int)rank * (a.nb / 2));
          if (++stage == (uint32_t)stages) { stage = 0; phase ^= 1; }
        }
      }
      __syncwarp();
    } else if (warp == 1) {
      // ------------------------------------------------ MMA issuer (leader CTA)
      if (rank == 0) {
        const uint32_t idesc = fc_idesc<ST>(a.nb);
        const bool leader = elect_one();
        mbar_wait(sbase + FC_SM_TEMPTY, (lt & 1) ^ 1);
        tc_fence_after();
        for (int kb = k0; kb < k1; ++kb) {
          mbar_wait(sbase + FC_SM_FULL + 8 * stage, phase);
          tc_fence_after();
          const uint32_t st0 = sbase + stage * sbytes;
          const uint64_t ad = umma_desc_sw128(st0), bd = umma_desc_sw128(st0 + FC_W_TILE);
          if (leader) {
            tc_mma<ST, 2>(tmem_base, ad, bd, idesc, kb > k0 ? 1u : 0u);
            tc_mma<ST, 2>(tmem_base, ad + 2, bd + 2, idesc, 1u);
            tc_mma<ST, 2>(tmem_base, ad + 4, bd + 4, idesc, 1u);
            tc_mma<ST, 2>(tmem_base, ad + 6, bd + 6, idesc, 1u);
            tc_commit<2>(sbase + FC_SM_EMPTY + 8 * stage);
          }
          __syncwarp();
          if (++stage == (uint32_t)stages) { stage = 0; phase ^= 1; }
        }
        if (leader) tc_commit<2>(sbase + FC_SM_TFULL);
        __syncwarp();
      }
    } else {
      // ------------------------------------------------ epilogue: TMEM -> y / partials
      // two warps per TMEM lane quarter (warp % 4), alternating 32-column chunks
      const int q = warp & 3, half = (warp - 2) >> 2;
      mbar_wait(sbase + FC_SM_TFULL, lt & 1);
      tc_fence_after();
      if (prof && t_full == 0) t_full = fc_gtimer();
      const int b0 = ch * a.nb;
      const int ncols = min(a.nb, a.B - b0);
      const bool partial = s > 1;
      const int n = rb * FC_ROWS + (int)rank * 128 + q * 32 + lane;
      const bool nok = n < a.N;
      const float bias = (!partial && nok) ? __ldg(&a.bias[n]) : 0.f;
      for (int c0 = 32 * half; c0 < ncols; c0 += 64) {         // warp-uniform
        uint32_t v[32];
        tmem_ld32(tmem_base + ((uint32_t)(q * 32) << 16) + c0, v);
        tmem_ld_wait();
        const int nc = min(32, ncols - c0);
        if (nok) {
          if (partial) {
            float *wsb = a.ws + ((size_t)split * a.B + b0 + c0) * a.N + n;
#pragma unroll
            for (int i = 0; i < 32; ++i)
              if (i < nc) wsb[(size_t)i * a.N] = __uint_as_float(v[i]);
          } else {
#pragma unroll
            for (int i = 0; i < 32; ++i)
              if (i < nc)
                fc_store(a.y, (size_t)(b0 + c0 + i) * a.ldy + n,
                         fc_act(__uint_as_float(v[i]) + bias, a.relu), a.out_mode);
          }
        }
      }
      tc_fence_before();
      __syncwarp();
      if (lane == 0) {
        if (rank == 0) mbar_arrive(sbase + FC_SM_TEMPTY);
        else mbar_arrive_cluster(mapa(sbase + FC_SM_TEMPTY, 0));
      }
      if (partial) {
        // meet the unit's other 2s - 1 CTAs, then reduce this CTA's row slice
        if (prof && t_st == 0) t_st = fc_gtimer();
        epi_bar();
        const int t = tid - 64;
        if (t == 0) {
          __threadfence();
          atomicAdd(&a.sem[u], 1u);
          while (ld_acquire(&a.sem[u]) < 2u * s) __nanosleep(64);
        }
        epi_bar();
        if (prof && t_met == 0) t_met = fc_gtimer();
        const int idx = split * 2 + (int)rank;
        if (s == 2) fc_reduce<2>(a, rb, ch, idx, t);
        else if (s == 4) fc_reduce<4>(a, rb, ch, idx, t);
        else if (s == 8) fc_reduce<8>(a, rb, ch, idx, t);
        else fc_reduce<16>(a, rb, ch, idx, t);
        epi_bar();
        if (prof && t_red == 0) t_red = fc_gtimer();
        if (t == 0) {   // the last CTA out re-arms the unit's counters for the next launch
          if (atomicAdd(&a.sem[a.units + u], 1u) == 2u * s - 1) {
            a.sem[u] = 0;
            a.sem[a.units + u] = 0;
          }
        }
      }
    }
  }
  tc_fence_before();
  __syncthreads();
  cluster_sync();
  tc_fence_after();
  if (prof && warp == 2 && lane == 0) {
    const unsigned long long t_exit = fc_gtimer();
    atomicAdd(&g_fc_prof[0], t_wait - t_entry);
    atomicAdd(&g_fc_prof[1], t_full - t_wait);
    atomicAdd(&g_fc_prof[2], (t_st ? t_st : t_full) - t_wait);
    atomicAdd(&g_fc_prof[3], (t_met ? t_met : t_full) - t_wait);
    atomicAdd(&g_fc_prof[4], (t_red ? t_red : t_full) - t_wait);
    atomicAdd(&g_fc_prof[5], t_exit - t_wait);
    atomicAdd(&g_fc_prof[6], 1ULL);
    atomicMax(&g_fc_prof[7], ~t_entry);
    atomicMax(&g_fc_prof[8], t_exit);
    atomicMax(&g_fc_prof[9], ~t_wait);
  }
  if (warp == 1)
    asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, %1;" ::"r"(tmem_base),
                 "r"(a.tmem_cols));
}

template <int ST>
static cudaError_t fc_launch(const CUtensorMap *tw, const CUtensorMap *tx, const FcArgs &args,
                             int grid, cudaStream_t s) {
  static bool attr = false;
  if (!attr) {
    cudaError_t e = cudaFuncSetAttribute(fc_tc_kernel<ST>,
                                         cudaFuncAttributeMaxDynamicSharedMemorySize,
                                         (int)FC_SMEM_BYTES);
    if (e != cudaSuccess) return e;
    attr = true;
  }
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(grid);
  cfg.blockDim = dim3(FC_THREADS);
  cfg.dynamicSmemBytes = FC_SMEM_BYTES;
  cfg.stream = s;
  cudaLaunchAttribute attr_[2];
  attr_[0].id = cudaLaunchAttributeClusterDimension;      // the CTA pair
  attr_[0].val.clusterDim.x = 2;
  attr_[0].val.clusterDim.y = 1;
  attr_[0].val.clusterDim.z = 1;
  attr_[1].id = cudaLaunchAttributeProgrammaticStreamSerialization;   // PDL
  attr_[1].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr_;
  cfg.numAttrs = 2;
  return cudaLaunchKernelEx(&cfg, fc_tc_kernel<ST>, *tw, *tx, args);
}

int fc_stage_count(int nb) {
  const int per = FC_W_TILE + nb / 2 * 128;
  return std::min(FC_MAX_STAGES, FC_STAGE_BUDGET / per);
}

// Debug: the FC timeline counters (prof build)
cudaError_t fc_profile(int reset, unsigned long long out[16]) {
  cudaError_t e = cudaDeviceSynchronize();
  if (e != cudaSuccess) return e;
  if (out) e = cudaMemcpyFromSymbol(out, g_fc_prof, sizeof(unsigned long long) * 16);
  if (e != cudaSuccess) return e;
  if (reset) {
    unsigned long long z[16] = {};
    e = cudaMemcpyToSymbol(g_fc_prof, z, sizeof(z));
  }
  return e;
}

cudaError_t launch_fc_tc(const FcPlan &p, int st, const CUtensorMap *tmap_w,
                         const CUtensorMap *tmap_x, const float *bias, void *y, float *ws,
                         unsigned *sem, int N, int B, int kblocks, int relu, int out_mode,
                         int ldy, const Budget &b, cudaStream_t s) {
  if (p.splits < 1 || p.splits > 16 || (p.splits & (p.splits - 1)) || p.nb < 16 || p.nb > 256 ||
      p.nb % 16 || (p.splits > 1 && (!ws || !sem)) || p.grid != 2 * p.splits * p.groups)
    return cudaErrorInvalidValue;
  FcArgs a;
  static const int prof_env = [] {
    const char *e = exp_env("PCNN_TC_PROFILE");
    return e && e[0] == '1' ? 1 : 0;
  }();
  a.prof = prof_env;
  a.N = N;
  a.B = B;
  a.kblocks = kblocks;
  a.kbps = p.kbps;
  a.splits = p.splits;
  a.nb = p.nb;
  a.rblocks = p.rblocks;
  a.chunks = p.chunks;
  a.units = p.rblocks * p.chunks;
  a.groups = p.groups;
  a.stages = fc_stage_count(p.nb);
  if (const char *e = exp_env("PCNN_FC_STAGES"))      // experiments build only
    a.stages = std::max(2, std::min(a.stages, atoi(e)));
  a.stage_bytes = FC_W_TILE + p.nb / 2 * 128;
  int cols = 32;
  while (cols < p.nb) cols <<= 1;
  a.tmem_cols = cols;
  a.kbe = st == ST_BF16 ? 64 : 32;
  a.relu = relu;
  a.out_mode = out_mode;
  a.ldy = ldy;
  a.y = y;
  a.ws = ws;
  a.sem = sem;
  a.bias = bias;
  a.b = b;
  if (a.stages < 2) return cudaErrorInvalidValue;
  cudaError_t e = st == ST_BF16 ? fc_launch<ST_BF16>(tmap_w, tmap_x, a, p.grid, s)
                                : fc_launch<ST_F32>(tmap_w, tmap_x, a, p.grid, s);
  if (e != cudaSuccess) return e;
  return cudaGetLastError();
}

}  // namespace pcnn
