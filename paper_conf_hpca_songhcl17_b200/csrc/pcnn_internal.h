// pcnn_internal.h -- shared declarations of the runtime and its kernels.
// Part of libpcnn.so (the CUDA product path).  Never includes oracle/.
#pragma once

#include <cuda.h>
#include <cuda_runtime.h>
#include <cuda_bf16.h>
#include <stdint.h>
#include <stdlib.h>

// Tuning / A-B experiment switches (PCNN_STAGES, PCNN_TC_SKIP, PCNN_FORCE_*,
// PCNN_LRN_*, ...) are read from the environment ONLY in the experiments
// build (python -m paper_conf_hpca_songhcl17_b200.build --prof, which defines
// PCNN_EXPERIMENTS=1 and writes build/prof/libpcnn_prof.so).  In the shipped
// libpcnn.so exp_env() is always nullptr: no environment variable can skip
// work, change a plan or select another kernel.  Supported layout choices are
// pcnn_net_desc.flags and pcnn_set_layer_plan (include/pcnn.h).
#ifndef PCNN_EXPERIMENTS
#define PCNN_EXPERIMENTS 0
#endif

namespace pcnn {

inline const char *exp_env(const char *name) {
#if PCNN_EXPERIMENTS
  return getenv(name);
#else
  (void)name;
  return nullptr;
#endif
}

constexpr int kMaxSMs = 256;          // census mask width

// ---------------------------------------------------------------- PDL
// Every kernel of the hot path is launched with programmatic stream
// serialization (programmatic dependent launch): its CTAs may be scheduled
// while the previous kernel of the stream is still running.  Each kernel
// (1) executes griddepcontrol.wait before it reads any activation or writes
// any global memory -- the wait returns once every prerequisite grid has
// completed and its writes are visible -- and (2) executes
// griddepcontrol.launch_dependents once all of its CTAs are resident, so the
// next kernel's launch latency, CTA rasterisation and prologue (barrier init,
// TMEM allocation, tensor-map prefetch, weight prefetch) overlap this
// kernel's tail.  Only read-only constants (weights, bias, tap tables) may be
// touched before the wait.
#ifdef __CUDACC__
__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
__device__ __forceinline__ void pdl_trigger() {
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
}
// the common case: nothing to prefetch
__device__ __forceinline__ void pdl_enter() {
  pdl_wait();
  pdl_trigger();
}
#endif

template <typename... KArgs, typename... Args>
inline cudaError_t launch_pdl(void (*kernel)(KArgs...), dim3 grid, dim3 block, size_t smem,
                              cudaStream_t s, Args &&...args) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = grid;
  cfg.blockDim = block;
  cfg.dynamicSmemBytes = smem;
  cfg.stream = s;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  return cudaLaunchKernelEx(&cfg, kernel, static_cast<KArgs>(args)...);
}

// Element storage types of activations / packed weights.
enum StoreType : int { ST_F32 = 0, ST_BF16 = 1 };
// Epilogue output modes.
enum OutMode : int { OUT_BF16 = 0, OUT_F32_TF32 = 1, OUT_F32 = 2 };

// SM / CTA budget handed to every layer kernel (P:213 PSM).
//   gated == 0 : no budget (static schedule over all SMs)
//   gated == 1 : CTA admitted iff %smid < n_sms and fewer than tlp CTAs of
//                this launch were admitted on its SM; admitted CTAs pull
//                tiles from an atomic counter (ctr[0]).  ctr[1 + smid] counts
//                admissions.  ctr must be zeroed before the launch.
struct Budget {
  int gated;
  int n_sms;
  int tlp;
  int pad_;
  unsigned long long *ctr;
  unsigned int *census;   // 8 words or nullptr
};

// Implicit-GEMM convolution geometry (one launch, all groups).
// GEMM per group g:  O[M x Nfg] = A[M x K] * B_g[Nfg x K]^T  with
//   M = B*Ho*Wo output pixels, A = im2col(X) (never materialised),
//   K ordered (r, s, c) over the Cg stored channels of group g.
struct ConvGeom {
  int M;            // B*Ho*Wo
  int H, W, Cs;     // input spatial size, stored channels per pixel
  int Cg;           // stored channels per group read by the GEMM
  int S, stride, pad;
  int Ho, Wo;
  int Nfg;          // output channels per group
  int groups;
  int out_cs;       // output pixel stride in elements (channels stored)
  int K;            // S*S*Cg
  int Kpad;         // K rounded up to the kernel's K-block
  int relu;
  int out_mode;     // OutMode
  // padded-layout ("shifted window") mode, tcgen05 only (pm = 1): input and
  // output share one zero-haloed grid hv x wv per image, M = B*hv*wv virtual
  // rows, and the A rows of tap (r, s) for output row i are input rows
  // i + (r - pad)*wv + (s - pad).  Rows outside the valid window
  // [vh, vh + Ho) x [vh, vh + Wo) are written as zeros (they are the next
  // layer's padding).  The runtime uses the shared-halo grid (vh = 0,
  // hv = H + h, wv = W + h): the h zero columns after one row are the left
  // padding of the next, the h zero rows after one image the top padding of
  // the next (the first image's top padding is TMA's out-of-bounds zero fill).
  // Requires stride 1 and S == 2*pad + 1.
  int pm;
  int hv, wv, vh;
  // perforated variant (NEXT-1, reading R13; im2col mode only): the GEMM rows
  // are the kept output positions of a psh x psw grid (Ho, Wo above are the
  // kept counts), i.e. input windows stride*psh / stride*psw apart; ih = zero
  // halo of the stored input (shared-halo grid [B][H + ih][W + ih][Cs],
  // interior at the origin); 0 = plain
  int psh, psw, ih;
  // row-perforated padded mode (pm = 2): the kept output rows p' (p = psh p')
  // of each image form segments of wv virtual rows; a CTA tile is nseg
  // consecutive kept rows of one image (nseg * wv <= 128 MMA rows), tpi tiles
  // per image, hk kept rows per image; M = B * tpi * 128.  The output is the
  // compact kept grid [B][hk][Wo][out_cs].
  int nseg, tpi, hk;
  // real (unpadded) channels per group, 0 = Cg: padded-layout UMMAs over the
  // zero channel padding of the last slab are skipped (their products are 0)
  int Creal;
};

// ---------------------------------------------------------------- launchers
// All return cudaSuccess or the launch error; they never synchronise.

// a1: NCHW fp32 [B][C][H][W] -> NHWC storage [B][Hs][Ws][Cs]; blk > 1 is
// space-to-depth by blk with the conv's padding `pad` folded in.
cudaError_t launch_stage_input(const float *x, void *y, int st, int B, int C,
                               int H, int W, int Hs, int Ws, int Cs, int blk,
                               int pad, int tf32_round, cudaStream_t s);
// a1 for a first conv with 3 input channels and S*S*3 <= 128: writes the
// conv's im2col rows [B][Ho + 2h][Wo + 2h][Kp] (interior of a halo-h grid;
// h = 0: compact) so the conv runs as a 1x1 conv.
cudaError_t launch_stage_im2col(const float *x, void *y, int st, int B, int C, int H,
                                int W, int S, int stride, int pad, int Ho, int Wo,
                                int Kp, int halo, int tf32_round, cudaStream_t s);
// final NHWC storage -> NCHW fp32 flatten
cudaError_t launch_unstage_output(const void *x, int st, float *y, int B,
                                  int C, int H, int W, int Cs, cudaStream_t s);

// FP32 SIMT implicit-GEMM conv / FC (check path, K3).
cudaError_t launch_conv_simt(const ConvGeom &g, const float *x,
                             const float *w, const float *bias, float *y,
                             const int *ktab, const Budget &b, int grid,
                             cudaStream_t s);
int conv_simt_tiles(const ConvGeom &g);
void conv_simt_tile_shape(int *tm, int *tn);

// tcgen05 implicit-GEMM conv / FC (K1/K2).
struct TcPlan {
  int cg;          // CTAs per tile: 1 (M = 128) or 2 (CTA pair, M = 256)
  int bn;          // N tile (16..256, multiple of 16)
  int mtiles, ntiles, tiles;   // output tiles (eq. 4 grid size)
  int splits;      // split-K factor (1 = none); chosen from the shape only
  int kb_per_split;
  int units;       // tiles * splits work units
  int grid;        // CTAs = cg * min(units, SM budget / cg)
  int rect_w, rect_h, rect_n;  // 0 = im2col A tiles; else rectangle tiles (tiled TMA)
  int a_stages, b_stages;      // padded mode: A (row-window) and B (tap slab) ring depths
  int msub;                    // padded mode: 128-row M sub-tiles per CTA sharing each B slab
  int ww;                      // padded mode: whole-slab A windows (all S x S taps; no split-K)
  double unit_us;              // modelled time of one work unit on its SM(s) (eq. 12 per wave)
};
// Launches the GEMM and, when p.splits > 1, the deterministic split-K
// reduction (ws must hold splits * M * out_cs floats; a split-K output must
// be packed, out_cs == groups * Nfg, with out_cs % 4 == 0).
// tmap_x: TMA im2col map of the NHWC input ({Cs, W, H, N}, corners -pad /
// pad-(S-1), channelsPerPixel = slab, 128 pixels per column, swizzle =
// slab bytes); tmap_w: tiled map of the packed weights (box 64|32 x bn/cg).
cudaError_t launch_conv_tc(const ConvGeom &g, int st, const CUtensorMap *tmap_x,
                           const CUtensorMap *tmap_w, const float *bias,
                           void *y, const int *ktab, const TcPlan &p, float *ws,
                           const Budget &b, cudaStream_t s, const float *lrn = nullptr,
                           const CUtensorMap *tmap_y = nullptr,
                           const CUtensorMap *tmap_y64 = nullptr);
// tmap_y (optional): tiled map of the output [M][out_cs] (box 32 columns x
// 32 rows, SW64 for bf16 / SW128 for fp32); full 32-column chunks are then
// written by TMA tensor stores from the epilogue's staging boxes.
// tmap_y64 (optional, bf16 output): the same matrix with 64-column boxes
// (128 B rows, SW128), used for full 64-column chunks.
// lrn (optional) = {size, alpha, beta, k} of a following LRN layer fused into
// the epilogue (size 5, one N tile holding all channels, no split-K).
// A-slab width in bytes (128 / 64 / 32) for Cg channels per group, 0 if the
// group width is not a multiple of 32 bytes.
int tc_slab_bytes(int st, int cg_channels);
int tc_stages_for(int bn, int cg);
// padded mode: ring depths for an N tile, CTA grouping, slab width and kernel size
void tc_pm_stages(int bn, int cg, int slab_bytes, int S, int msub, int *a_stages,
                  int *b_stages, int rows, int ww);
// padded mode: A window rows per sub-tile, per filter row (ww = 0) or whole
// (ww = 1: 128 + (S - 1)(wv + 1) rows feed all S x S taps)
int pm_window_rows(int S, int wv, int ww);
// debug: per-role barrier-wait cycle totals accumulated while PCNN_TC_PROFILE=1
cudaError_t tc_profile(int reset, unsigned long long out[32]);
int tc_block_k_elems(int st);          // K-block in elements (128 B)
cudaError_t tc_init();                 // sets the kernels' smem attributes
size_t tc_smem_bytes();
int tc_max_ktab();

// a6: weight-streaming FC (kernels_fc.cu).  A CTA pair (cta_group::2) owns
// 256 weight rows (the UMMA M) for nb images of a batch chunk (the UMMA N);
// `splits` pairs split K in fixed, batch-independent ranges of kbps K-blocks
// and reduce their FP32 partials in split order.
struct FcPlan {
  int splits;     // K split = CTA pairs per unit (power of two, <= 16)
  int kbps;       // K-blocks per split
  int nb;         // batch columns per chunk (16..256, multiple of 16)
  int rblocks;    // ceil(N / 256)
  int chunks;     // ceil(B / nb)
  int groups;     // concurrent unit workers (each = splits CTA pairs)
  int grid;       // CTAs = 2 x splits x groups
  double unit_us; // modelled time of one split of one unit on its CTA pair
};
int fc_stage_count(int nb);
// uint8 NCHW pixels -> fp32 network input (pixel - mean[c]) * scale
cudaError_t launch_pixels_u8(const unsigned char *px, const float *mean, float scale, float *y,
                             int B, int C, int HW, cudaStream_t s);
cudaError_t fc_profile(int reset, unsigned long long out[16]);   // debug timeline (prof build)
// tmap_w: 4-D map of the re-tiled weights [RB][KB][128][128 B] (box = one
// 16 KB tile, SW128); tmap_x: tiled map of the input [B][K] (box 128 B x
// nb / 2 rows, SW128); y: [B][ldy] output; ws: splits * B * N floats and sem:
// 2 * units zeroed counters when splits > 1.
cudaError_t launch_fc_tc(const FcPlan &p, int st, const CUtensorMap *tmap_w,
                         const CUtensorMap *tmap_x, const float *bias, void *y, float *ws,
                         unsigned *sem, int N, int B, int kblocks, int relu, int out_mode,
                         int ldy, const Budget &b, cudaStream_t s);

// a4 / a5: LRN (lrn_size > 0) followed by pooling (k x k, stride s; k = s =
// 1 for no pooling), NHWC with C stored input channels.  out_groups > 0
// writes the output with each of the out_groups channel groups padded to
// out_cg_pad channels (zeros), the layout a following grouped conv loads
// with full 128-byte TMA slabs.  in_halo / out_halo: zero border width of
// the input / output layouts ([B][H + 2h][W + 2h][C]); the kernel writes the
// output border zeros itself.
cudaError_t launch_lrn_pool(const void *x, void *y, int st, int tf32_round, int B,
                            int H, int W, int C, int lrn_size, float alpha,
                            float beta, float kk, int k, int s, int is_max,
                            int Ho, int Wo, int out_groups, int out_cg_pad,
                            int in_halo, int out_halo, const Budget &b, int grid,
                            cudaStream_t stream);
long long lrn_pool_tiles(int st, int B, int W, int C, int lrn, int k, int s,
                         int Ho, int Wo);
int lrn_pool_occupancy(int st);
// NEXT-1 interpolation: y [B][Ho + 2ho][Wo + 2ho][Cs] from the kept grid
// t [B][ceil(Ho/sh)][ceil(Wo/sw)][Cs] by nearest kept neighbour (ties to the
// lower index, reading R13); halo cells written as zeros.
cudaError_t launch_perf_interp(const void *t, void *y, int st, int B, int Ho, int Wo, int sh,
                               int sw, int Cs, int ho, cudaStream_t s);
// a7
cudaError_t launch_softmax_entropy(const float *z, float *p, float *h, int B,
                                   int N, cudaStream_t s);

// occupancy helpers for gated launches
int simt_conv_occupancy();

}  // namespace pcnn
