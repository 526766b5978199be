// runtime.cu -- libpcnn host runtime and C ABI (include/pcnn.h).
//
// Responsibilities: validate layer descriptors, infer shapes, pack weights
// into the kernels' K-major (r, s, c) layouts in the storage precision, own
// the activation arena, plan each layer (engine, tile, grid, SM budget), run
// the rank-r variant's SVD, and enqueue the hot path (optionally through a
// cached CUDA graph).  No arithmetic of the hot path runs on the host.
#include <cudaTypedefs.h>

#include <algorithm>
#include <cmath>
#include <cstdio>
#include <cstring>
#include <map>
#include <memory>
#include <mutex>
#include <string>
#include <tuple>
#include <vector>

#include "../../include/pcnn.h"
#include "pcnn_internal.h"
#include "svd.h"

using namespace pcnn;

// ------------------------------------------------------------------ errors
static thread_local std::string g_err;

static pcnn_status fail(pcnn_status s, const std::string &msg) {
  g_err = msg;
  return s;
}

#define CUDA_TRY(expr)                                                          \
  do {                                                                          \
    cudaError_t e_ = (expr);                                                    \
    if (e_ != cudaSuccess)                                                      \
      return fail(PCNN_ERR_CUDA, std::string(#expr) + ": " + cudaGetErrorString(e_)); \
  } while (0)

// every kernel launch of the hot path goes through this counter
static thread_local int g_launches = 0;
static inline cudaError_t counted(cudaError_t e) {
  ++g_launches;
  return e;
}

// ------------------------------------------------------------------ host rounding
static inline uint16_t f32_to_bf16_rne(float f) {
  uint32_t u;
  std::memcpy(&u, &f, 4);
  if ((u & 0x7F800000u) == 0x7F800000u) return (uint16_t)(u >> 16);  // inf/nan
  u += 0x7FFFu + ((u >> 16) & 1u);
  return (uint16_t)(u >> 16);
}
static inline float tf32_rna_host(float f) {
  uint32_t u;
  std::memcpy(&u, &f, 4);
  if ((u & 0x7F800000u) != 0x7F800000u) {
    u += 0x1000u;
    u &= 0xFFFFE000u;
  }
  float r;
  std::memcpy(&r, &u, 4);
  return r;
}

// ------------------------------------------------------------------ driver entry
static PFN_cuTensorMapEncodeIm2col_v12000 get_encode_im2col() {
  static PFN_cuTensorMapEncodeIm2col_v12000 fn = nullptr;
  static std::once_flag once;
  std::call_once(once, [] {
    void *p = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeIm2col", &p, cudaEnableDefault, &q) ==
            cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = (PFN_cuTensorMapEncodeIm2col_v12000)p;
  });
  return fn;
}

static PFN_cuTensorMapEncodeTiled_v12000 get_encode_tiled() {
  static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
  static std::once_flag once;
  std::call_once(once, [] {
    void *p = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) ==
            cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = (PFN_cuTensorMapEncodeTiled_v12000)p;
  });
  return fn;
}

// ------------------------------------------------------------------ net state
namespace {

struct GemmStage {           // one implicit-GEMM launch
  ConvGeom g{};              // M filled per batch
  int in_c = 0, in_h = 0, in_w = 0;
  int st = ST_F32;           // storage type of input / weights
  int engine = 0;            // 0 SIMT, 1 tcgen05
  bool is_fc = false;        // FC layer (tcgen05: the weight-streaming FC kernel)
  unsigned *d_sem = nullptr; // FC split-K arrival counters (2 x units, zero at rest)
  int sem_count = 0;
  void *d_w = nullptr;       // packed [groups*Nfg][Kpad]
  float *d_bias = nullptr;
  int *d_ktab = nullptr;     // per-element (r,s,c) table
  std::map<int, CUtensorMap> tmaps;  // weight maps by box rows
  std::map<std::tuple<const void *, int, int, int, int>, CUtensorMap> xmaps;   // A maps by
                                                 // (input, batch, rect w, h, n)
  // output maps by (y, M): 32-column boxes, and 64-column boxes (bf16)
  std::map<std::pair<const void *, long long>, std::pair<CUtensorMap, CUtensorMap>> ymaps;
  size_t w_bytes = 0;
  void release() {
    if (d_w) cudaFree(d_w);
    if (d_bias) cudaFree(d_bias);
    if (d_ktab) cudaFree(d_ktab);
    if (d_sem) cudaFree(d_sem);
    d_sem = nullptr;
    sem_count = 0;
    d_w = nullptr;
    d_bias = nullptr;
    d_ktab = nullptr;
    tmaps.clear();
    xmaps.clear();
    ymaps.clear();
  }
};

struct Layer {
  pcnn_layer_desc d{};
  int in_c = 0, in_h = 0, in_w = 0, in_cs = 0;
  int out_c = 0, out_h = 0, out_w = 0, out_cs = 0;
  int gemm = 0;             // conv or fc
  GemmStage exact;
  // rank-r variant
  int variant = PCNN_VARIANT_EXACT, rank = 0;
  GemmStage r1, r2;
  // perforated variant (NEXT-1): kept-grid steps (1, 1 = off) and its stage
  int perf_sh = 1, perf_sw = 1;
  GemmStage pf;
  std::vector<float> host_w;   // OIHW copy kept for the SVD (conv only)
  std::vector<Svd> svd;        // per group (lazily computed)
  // budget
  int n_sms = 0, tlp = 0;
  // tile-choice override (pcnn_set_layer_plan; 0 = planner's choice)
  int plan_cg = 0, plan_msub = 0;
  int out_groups = 0, out_cg_pad = 0;    // padded-group output layout (lrn/pool)
  // zero border (halo) of the stored input / output activation; pm_halo > 0:
  // this conv runs in padded-layout mode (ConvGeom::pm) with that halo
  int in_halo = 0, out_halo = 0, pm_halo = 0;
  unsigned long long *d_ctr = nullptr;   // 3 launch slots x (1 + kMaxSMs)
  unsigned int *d_census = nullptr;      // 8 words
};

}  // namespace

struct pcnn_net {
  pcnn_net_desc desc{};
  int device = 0;
  int num_sms = 148;
  int st = ST_F32;
  int in_cs = 4;
  std::vector<Layer> layers;
  size_t act_bytes = 0;     // per arena buffer
  void *d_act[3] = {nullptr, nullptr, nullptr};
  float *d_host_in = nullptr, *d_host_out = nullptr, *d_host_p = nullptr,
        *d_host_h = nullptr;
  unsigned char *d_host_u8 = nullptr;   // pcnn_infer_host_u8 pixels
  float *d_mean = nullptr;              // per-channel mean (C floats)
  // pcnn_infer_host pipelining: host->device copies of later chunks on their
  // own stream while earlier chunks compute
  cudaStream_t copy_stream = nullptr;
  cudaEvent_t ev_copy[5] = {nullptr, nullptr, nullptr, nullptr, nullptr};
  int out_elems = 0;
  int occ_simt = 1, occ_lp = 1;
  // input staging geometry (space-to-depth by `blk` for a strided first conv)
  int stage_h = 0, stage_w = 0, stage_blk = 1, stage_pad = 0, stage_c = 0;
  int stage_im2col = 0;     // 1: layer 0 input staged as im2col rows (1x1 conv)
  bool fuse_lrn_pool = true;
  bool conv_lrn_pm = false;    // PCNN_FLAG_CONV_LRN_EPILOGUE
  bool per_row_windows = false; // PCNN_FLAG_PER_ROW_WINDOWS
  bool perf_im2col = false;    // PCNN_FLAG_PERFORATION_IM2COL
  bool census = false;
  // CUDA graph cache
  uint64_t version = 1;
  struct GraphKey {
    int batch;
    const void *in, *out, *p, *h;
    cudaStream_t s;
    uint64_t version;
    bool operator<(const GraphKey &o) const {
      return std::tie(batch, in, out, p, h, s, version) <
             std::tie(o.batch, o.in, o.out, o.p, o.h, o.s, o.version);
    }
  };
  std::map<GraphKey, cudaGraphExec_t> graphs;
  bool use_graphs = true;
  int launches_per_infer = 0;
  float *d_ws = nullptr;    // split-K partials
  size_t ws_bytes = 0;
  // live per-layer timing (pcnn_set_layer_timing)
  bool timing = false;
  std::vector<std::vector<cudaEvent_t>> timing_sets;   // recorded, unread
  std::vector<std::vector<cudaEvent_t>> timing_free;   // reusable
};

// ------------------------------------------------------------------ geometry
static int conv_out(int in, int k, int st, int pad) {
  if (st <= 0 || in + 2 * pad < k) return -1;
  return (in + 2 * pad - k) / st + 1;
}
static int pool_out(int in, int k, int st) {
  if (st <= 0 || in < k) return -1;
  int o = (in - k + st - 1) / st + 1;
  if ((o - 1) * st >= in) --o;
  return o;
}
static int round_up(int a, int b) { return (a + b - 1) / b * b; }
static int esz_of(int st) { return st == ST_BF16 ? 2 : 4; }

static int storage_of(int precision) {
  return precision == PCNN_BF16 ? ST_BF16 : ST_F32;
}
static int chunk_elems(int precision) {
  // channel padding unit of stored activations: 32 B, the narrowest TMA
  // im2col slab of the tcgen05 path
  return precision == PCNN_BF16 ? 16 : 8;
}

// Shape inference over the descriptor list (host only).  Fills in/out dims.
static pcnn_status infer_shapes(const pcnn_net_desc *d, const pcnn_layer_desc *L, int n,
                                std::vector<Layer> &out) {
  if (!d || !L || n <= 0) return fail(PCNN_ERR_INVALID_ARGUMENT, "null descriptor or no layers");
  if (d->in_channels <= 0 || d->in_height <= 0 || d->in_width <= 0)
    return fail(PCNN_ERR_SHAPE, "bad input shape");
  if (d->precision < PCNN_FP32_SIMT || d->precision > PCNN_BF16)
    return fail(PCNN_ERR_INVALID_ARGUMENT, "bad precision");
  const int ch = chunk_elems(d->precision);
  out.assign(n, Layer());
  int c = d->in_channels, h = d->in_height, w = d->in_width;
  int cs = round_up(c, ch);
  for (int i = 0; i < n; ++i) {
    Layer &ly = out[i];
    ly.d = L[i];
    ly.in_c = c;
    ly.in_h = h;
    ly.in_w = w;
    ly.in_cs = cs;
    const auto &li = L[i];
    char buf[160];
    switch (li.kind) {
      case PCNN_CONV: {
        const int g = li.groups <= 0 ? 1 : li.groups;
        ly.d.groups = g;
        if (li.out_channels <= 0 || li.kernel <= 0 || li.stride <= 0 || li.pad < 0 ||
            c % g || li.out_channels % g) {
          snprintf(buf, sizeof buf, "layer %d: bad conv descriptor", i);
          return fail(PCNN_ERR_SHAPE, buf);
        }
        if (li.kernel > 255) return fail(PCNN_ERR_UNSUPPORTED, "kernel > 255");
        if (i == 0 && g > 1 && cs != c)
          return fail(PCNN_ERR_UNSUPPORTED, "grouped first layer needs C multiple of 8");
        const int ho = conv_out(h, li.kernel, li.stride, li.pad);
        const int wo = conv_out(w, li.kernel, li.stride, li.pad);
        if (ho <= 0 || wo <= 0) {
          snprintf(buf, sizeof buf, "layer %d: conv output empty", i);
          return fail(PCNN_ERR_SHAPE, buf);
        }
        ly.gemm = 1;
        c = li.out_channels;
        h = ho;
        w = wo;
        break;
      }
      case PCNN_FC:
        if (li.out_channels <= 0) return fail(PCNN_ERR_SHAPE, "bad fc descriptor");
        ly.gemm = 1;
        ly.d.groups = 1;
        c = li.out_channels;
        h = 1;
        w = 1;
        break;
      case PCNN_LRN:
        if (li.kernel <= 0 || (li.kernel % 2) == 0)
          return fail(PCNN_ERR_SHAPE, "LRN size must be odd");
        if (li.kernel > 9) return fail(PCNN_ERR_UNSUPPORTED, "LRN local size > 9");
        break;
      case PCNN_MAXPOOL:
      case PCNN_AVGPOOL: {
        const int ho = pool_out(h, li.kernel, li.stride);
        const int wo = pool_out(w, li.kernel, li.stride);
        if (li.kernel <= 0 || ho <= 0 || wo <= 0) return fail(PCNN_ERR_SHAPE, "bad pool");
        h = ho;
        w = wo;
        break;
      }
      default:
        return fail(PCNN_ERR_INVALID_ARGUMENT, "unknown layer kind");
    }
    ly.out_c = c;
    ly.out_h = h;
    ly.out_w = w;
    // stored channels: GEMM outputs keep exactly out_c (must be chunk-aligned to
    // feed the next GEMM); pool / LRN keep their input's storage.
    ly.out_cs = ly.gemm ? c : cs;
    cs = ly.out_cs;
  }
  return PCNN_OK;
}

static double layer_flops_exact(const Layer &ly, int B) {
  const auto &d = ly.d;
  if (d.kind == PCNN_CONV)
    return 2.0 * B * (double)ly.out_h * ly.out_w * d.out_channels *
           ((double)d.kernel * d.kernel * (ly.in_c / d.groups));   // eq. 1
  if (d.kind == PCNN_FC)
    return 2.0 * B * (double)d.out_channels * ((double)ly.in_c * ly.in_h * ly.in_w);
  return 0.0;
}

static double layer_flops_variant(const Layer &ly, int B) {
  if (ly.variant == PCNN_VARIANT_RANK && ly.d.kind == PCNN_FC)   // 2 B r (K + N)
    return 2.0 * B * ly.rank * ((double)ly.in_c * ly.in_h * ly.in_w + ly.d.out_channels);
  if (ly.perf_sh * ly.perf_sw > 1)       // eq. 1 FLOPs at the kept positions only
    return layer_flops_exact(ly, B) * ((ly.out_h + ly.perf_sh - 1) / ly.perf_sh) *
           ((ly.out_w + ly.perf_sw - 1) / ly.perf_sw) / ((double)ly.out_h * ly.out_w);
  if (ly.variant != PCNN_VARIANT_RANK) return layer_flops_exact(ly, B);
  const auto &d = ly.d;
  const double P = (double)B * ly.out_h * ly.out_w;
  const double K = (double)d.kernel * d.kernel * (ly.in_c / d.groups);
  const double Nfg = d.out_channels / d.groups;
  return 2.0 * P * ly.rank * (K + Nfg) * d.groups;
}

static double layer_bytes(const Layer &ly, int B, int precision, bool last) {
  const double e = precision == PCNN_BF16 ? 2.0 : 4.0;
  const double in = (double)B * ly.in_c * ly.in_h * ly.in_w * e;
  const double oe = last && ly.d.kind == PCNN_FC ? 4.0 : e;
  const double out = (double)B * ly.out_c * ly.out_h * ly.out_w * oe;
  double w = 0;
  if (ly.d.kind == PCNN_CONV)
    w = (double)ly.d.out_channels * (ly.in_c / ly.d.groups) * ly.d.kernel * ly.d.kernel * e;
  if (ly.d.kind == PCNN_FC) w = (double)ly.d.out_channels * ly.in_c * ly.in_h * ly.in_w * e;
  if (ly.variant == PCNN_VARIANT_RANK && ly.d.kind == PCNN_CONV) {
    const double K = (double)ly.d.kernel * ly.d.kernel * (ly.in_c / ly.d.groups);
    const double Nfg = ly.d.out_channels / ly.d.groups;
    w = (double)ly.d.groups * ly.rank * (K + Nfg) * e;
    // the stage-1 intermediate is written and read once
    w += 2.0 * B * ly.out_h * ly.out_w * (double)ly.d.groups * ly.rank * e;
  }
  return in + out + w;
}

// ------------------------------------------------------------------ packing
// F_m of Fig. 2 in the kernels' layout: row n = g*Nfg + f, column
// k = (r*S + s)*Cg_stored + c, zero for padded channels and k >= K.
static std::vector<float> pack_conv(const float *w, int Nf, int Cg_log, int Cg_st, int S,
                                    int Kpad) {
  std::vector<float> p((size_t)Nf * Kpad, 0.f);
  for (int n = 0; n < Nf; ++n)
    for (int c = 0; c < Cg_log; ++c)
      for (int r = 0; r < S; ++r)
        for (int s = 0; s < S; ++s)
          p[(size_t)n * Kpad + (size_t)(r * S + s) * Cg_st + c] =
              w[(((size_t)n * Cg_log + c) * S + r) * S + s];
  return p;
}

// FC weight [N][C*H*W] (C,H,W order) -> [N][Kpad] over the stored NHWC
// flatten (h, w, c_stored).
static std::vector<float> pack_fc(const float *w, int N, int C, int H, int W, int Cs,
                                  int Kpad) {
  std::vector<float> p((size_t)N * Kpad, 0.f);
  const size_t Kin = (size_t)C * H * W;
  for (int n = 0; n < N; ++n)
    for (int c = 0; c < C; ++c)
      for (int h = 0; h < H; ++h)
        for (int x = 0; x < W; ++x)
          p[(size_t)n * Kpad + ((size_t)h * W + x) * Cs + c] =
              w[(size_t)n * Kin + ((size_t)c * H + h) * W + x];
  return p;
}

static pcnn_status upload_weights(GemmStage &gs, const std::vector<float> &packed,
                                  int precision) {
  const size_t n = packed.size();
  if (precision == PCNN_BF16) {
    std::vector<uint16_t> b(n);
    for (size_t i = 0; i < n; ++i) b[i] = f32_to_bf16_rne(packed[i]);
    gs.w_bytes = n * 2;
    CUDA_TRY(cudaMalloc(&gs.d_w, gs.w_bytes));
    CUDA_TRY(cudaMemcpy(gs.d_w, b.data(), gs.w_bytes, cudaMemcpyHostToDevice));
  } else {
    std::vector<float> f(packed);
    if (precision == PCNN_TF32)
      for (auto &v : f) v = tf32_rna_host(v);
    gs.w_bytes = n * 4;
    CUDA_TRY(cudaMalloc(&gs.d_w, gs.w_bytes));
    CUDA_TRY(cudaMemcpy(gs.d_w, f.data(), gs.w_bytes, cudaMemcpyHostToDevice));
  }
  return PCNN_OK;
}

static int k_align(int precision) {
  if (precision == PCNN_BF16) return 64;   // one 128 B K-block
  if (precision == PCNN_TF32) return 32;
  return 16;                               // SIMT BK
}

// Build a GEMM stage.  w_oihw: [Nf][Cg_log][S][S]; for fc (is_fc) w is
// [N][C*H*W] and the geometry is a 1x1 conv on a 1x1 "image" of K features.
static pcnn_status build_stage(GemmStage &gs, const Layer &ly, int precision, int Nf,
                               int groups, int S, int stride, int pad, int relu,
                               int in_c, int in_h, int in_w, int in_cs, bool is_fc,
                               const float *w, const float *bias, int out_mode,
                               int pm_halo = 0, bool pm_valid = false) {
  gs.release();
  gs.st = storage_of(precision);
  gs.engine = precision == PCNN_FP32_SIMT ? 0 : 1;
  gs.is_fc = is_fc;
  gs.in_c = in_c;
  gs.in_h = in_h;
  gs.in_w = in_w;
  ConvGeom &g = gs.g;
  std::memset(&g, 0, sizeof g);
  const int ch = chunk_elems(precision);
  std::vector<float> packed;
  if (is_fc) {
    const int K = in_h * in_w * in_cs;
    g.H = g.W = 1;
    g.Cs = K;
    g.Cg = K;
    g.S = 1;
    g.stride = 1;
    g.pad = 0;
    g.Ho = g.Wo = 1;
    g.groups = 1;
    g.Nfg = Nf;
    g.K = K;
    g.Kpad = round_up(K, k_align(precision));
    packed = pack_fc(w, Nf, in_c, in_h, in_w, in_cs, g.Kpad);
  } else {
    const int Cg_log = in_c / groups;
    const int Cg_st = in_cs / groups;      // stored (possibly padded) channels per group
    if (gs.engine == 1 && tc_slab_bytes(gs.st, Cg_st) == 0)
      return fail(PCNN_ERR_UNSUPPORTED, "tcgen05 conv needs channels per group multiple of 32 bytes");
    g.H = in_h;
    g.W = in_w;
    g.Cs = in_cs;
    g.Cg = Cg_st;
    g.S = S;
    g.stride = stride;
    g.pad = pad;
    g.Ho = conv_out(in_h, S, stride, pad);
    g.Wo = conv_out(in_w, S, stride, pad);
    g.groups = groups;
    g.Nfg = Nf / groups;
    g.K = S * S * Cg_st;
    g.Kpad = round_up(g.K, k_align(precision));
    g.Creal = Cg_log;
    if (pm_halo > 0 && pm_valid) {
      // a 'valid' stride-1 conv (pad 0, S = 2h + 1) on its own input grid:
      // output (p, q) sits at grid row p*wv + q and reads input rows
      // (p + r)*wv + q + s; the output grid is the input grid, i.e. the
      // shared-halo layout of the output with halo S - 1 (layer 0 after
      // space-to-depth)
      if (gs.engine != 1 || stride != 1 || pad != 0 || S != 2 * pm_halo + 1)
        return fail(PCNN_ERR_UNSUPPORTED, "valid padded-layout mode needs pad 0, S = 2h + 1");
      g.pm = 1;
      g.vh = 0;
      g.hv = in_h;
      g.wv = in_w;
      g.pad = 0;
    } else if (pm_halo > 0) {
      // shared-halo grid: [H + h][W + h] per image, interior at
      // the origin; the zero columns / rows after a row / image are the left /
      // top padding of the next one
      if (gs.engine != 1 || stride != 1 || S != 2 * pad + 1 || pad > pm_halo)
        return fail(PCNN_ERR_UNSUPPORTED, "padded-layout mode needs a stride-1 'same' conv");
      g.pm = 1;
      g.vh = 0;
      g.hv = in_h + pm_halo;
      g.wv = in_w + pm_halo;
    }
    packed = pack_conv(w, Nf, Cg_log, Cg_st, S, g.Kpad);
    if (S > 1) {
      if (gs.engine == 1 && g.Kpad / ch > tc_max_ktab())
        return fail(PCNN_ERR_UNSUPPORTED, "conv K too large for the tap table");
      std::vector<int> tab(g.K);
      for (int k = 0; k < g.K; ++k) {
        const int tap = k / Cg_st, c = k % Cg_st;
        tab[k] = ((tap / S) << 24) | ((tap % S) << 16) | c;
      }
      CUDA_TRY(cudaMalloc(&gs.d_ktab, sizeof(int) * g.K));
      CUDA_TRY(cudaMemcpy(gs.d_ktab, tab.data(), sizeof(int) * g.K, cudaMemcpyHostToDevice));
    }
  }
  (void)ch;
  if (gs.engine == 1 && is_fc && tc_slab_bytes(gs.st, g.Cg) == 0)
    return fail(PCNN_ERR_UNSUPPORTED, "tcgen05 FC needs K multiple of 32 bytes");
  if (gs.engine == 1 && !is_fc && (g.Nfg % 8))
    return fail(PCNN_ERR_UNSUPPORTED, "tcgen05 conv needs N_f/g multiple of 8");
  g.relu = relu;
  g.out_mode = out_mode;
  g.out_cs = Nf;
  if (gs.engine == 1 && is_fc) {
    // weight-streaming FC: re-tile [N][Kpad] into contiguous 128-row x 128-B
    // K-block tiles, [row block][K-block][128 rows][128 B] (rows past N are
    // zeros), so every TMA box the kernel streams is one contiguous 16 KB run
    // of HBM instead of 128 rows 2*Kpad bytes apart
    const int kbe = k_align(precision) == 64 ? 64 : 32;
    const int KB = g.Kpad / kbe, RB = (Nf + 127) / 128;
    std::vector<float> t((size_t)RB * 128 * g.Kpad, 0.f);
    for (int n = 0; n < Nf; ++n)
      for (int kb = 0; kb < KB; ++kb)
        std::memcpy(&t[(((size_t)(n / 128) * KB + kb) * 128 + (n % 128)) * kbe],
                    &packed[(size_t)n * g.Kpad + (size_t)kb * kbe], sizeof(float) * kbe);
    packed.swap(t);
  }
  pcnn_status st = upload_weights(gs, packed, precision);
  if (st != PCNN_OK) return st;
  // zero-padded so the epilogue can read whole 32-column slices unguarded
  const size_t nb = (size_t)round_up(Nf, 256) + 256;
  std::vector<float> b(nb, 0.f);
  if (bias) std::memcpy(b.data(), bias, sizeof(float) * Nf);
  CUDA_TRY(cudaMalloc(&gs.d_bias, sizeof(float) * nb));
  CUDA_TRY(cudaMemcpy(gs.d_bias, b.data(), sizeof(float) * nb, cudaMemcpyHostToDevice));
  (void)ly;
  return PCNN_OK;
}

// Weight (B operand) map: boxes of `rows` filters x `slab` bytes of K.
static const CUtensorMap *stage_tmap(GemmStage &gs, int rows, int slab = 128) {
  const int bn = rows;
  const int key = rows * 1024 + slab;
  auto it = gs.tmaps.find(key);
  if (it != gs.tmaps.end()) return &it->second;
  auto enc = get_encode_tiled();
  if (!enc) return nullptr;
  CUtensorMap m;
  const int esz = esz_of(gs.st);
  const cuuint64_t dims[2] = {(cuuint64_t)gs.g.Kpad, (cuuint64_t)gs.g.Nfg * gs.g.groups};
  const cuuint64_t strides[1] = {(cuuint64_t)gs.g.Kpad * esz};
  const cuuint32_t box[2] = {(cuuint32_t)(slab / esz), (cuuint32_t)bn};
  const cuuint32_t estr[2] = {1, 1};
  const CUtensorMapSwizzle sw = slab == 128 ? CU_TENSOR_MAP_SWIZZLE_128B
                                : slab == 64 ? CU_TENSOR_MAP_SWIZZLE_64B
                                             : CU_TENSOR_MAP_SWIZZLE_32B;
  CUresult r = enc(&m, gs.st == ST_BF16 ? CU_TENSOR_MAP_DATA_TYPE_BFLOAT16 : CU_TENSOR_MAP_DATA_TYPE_FLOAT32,
                   2, gs.d_w, dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                   sw, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) return nullptr;
  return &(gs.tmaps[key] = m);
}

// TMA im2col map of a stage's NHWC input for `batch` images.
static const CUtensorMap *stage_xmap(GemmStage &gs, const void *x, int batch, const TcPlan &p) {
  // (padded-layout plans have no rectangle: rect_n carries the whole-window flag)
  const auto key = std::make_tuple(x, batch, p.rect_w, p.rect_h, gs.g.pm ? -1 - p.ww : p.rect_n);
  auto it = gs.xmaps.find(key);
  if (it != gs.xmaps.end()) return &it->second;
  const ConvGeom &g = gs.g;
  const int esz = esz_of(gs.st);
  const int slab = tc_slab_bytes(gs.st, g.Cg);
  CUtensorMap m;
  if (g.pm == 2) {
    // row-perforated padded layout: {channels, wv, grid rows} with the grid
    // rows traversed psh apart; a box is nseg kept rows of one filter row
    auto enct = get_encode_tiled();
    if (!enct) return nullptr;
    const cuuint64_t d3[3] = {(cuuint64_t)g.Cs, (cuuint64_t)g.wv, (cuuint64_t)batch * g.hv};
    const cuuint64_t s3[2] = {(cuuint64_t)g.Cs * esz, (cuuint64_t)g.wv * g.Cs * esz};
    const cuuint32_t box[3] = {(cuuint32_t)(slab / esz), (cuuint32_t)(g.wv + 2 * g.pad),
                               (cuuint32_t)(g.nseg * g.psh)};
    const cuuint32_t estr[3] = {1, 1, (cuuint32_t)g.psh};
    const CUtensorMapSwizzle sw = slab == 128 ? CU_TENSOR_MAP_SWIZZLE_128B
                                  : slab == 64 ? CU_TENSOR_MAP_SWIZZLE_64B
                                               : CU_TENSOR_MAP_SWIZZLE_32B;
    CUresult r = enct(&m, gs.st == ST_BF16 ? CU_TENSOR_MAP_DATA_TYPE_BFLOAT16
                                           : CU_TENSOR_MAP_DATA_TYPE_FLOAT32,
                      3, const_cast<void *>(x), d3, s3, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                      sw, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (r != CUDA_SUCCESS) return nullptr;
    if (gs.xmaps.size() > 64) gs.xmaps.clear();
    return &(gs.xmaps[key] = m);
  }
  if (g.pm) {
    // padded layout: the input is a plain [B*hv*wv][Cs] matrix; a box is the
    // (128 + S - 1)-row window of one filter row (rows outside the tensor --
    // the first / last window of the batch -- are zero-filled)
    auto enct = get_encode_tiled();
    if (!enct) return nullptr;
    const cuuint64_t d2[2] = {(cuuint64_t)g.Cs, (cuuint64_t)batch * g.hv * g.wv};
    const cuuint64_t s2[1] = {(cuuint64_t)g.Cs * esz};
    const cuuint32_t box[2] = {(cuuint32_t)(slab / esz), (cuuint32_t)pm_window_rows(g.S, g.wv, p.ww)};
    const cuuint32_t estr[2] = {1, 1};
    const CUtensorMapSwizzle sw = slab == 128 ? CU_TENSOR_MAP_SWIZZLE_128B
                                  : slab == 64 ? CU_TENSOR_MAP_SWIZZLE_64B
                                               : CU_TENSOR_MAP_SWIZZLE_32B;
    CUresult r = enct(&m, gs.st == ST_BF16 ? CU_TENSOR_MAP_DATA_TYPE_BFLOAT16
                                           : CU_TENSOR_MAP_DATA_TYPE_FLOAT32,
                      2, const_cast<void *>(x), d2, s2, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                      sw, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (r != CUDA_SUCCESS) return nullptr;
    if (gs.xmaps.size() > 64) gs.xmaps.clear();
    return &(gs.xmaps[key] = m);
  }
  const cuuint64_t dims[4] = {(cuuint64_t)g.Cs, (cuuint64_t)g.W, (cuuint64_t)g.H,
                              (cuuint64_t)batch};
  const cuuint64_t strides[3] = {(cuuint64_t)g.Cs * esz, (cuuint64_t)g.W * g.Cs * esz,
                                 (cuuint64_t)g.H * g.W * g.Cs * esz};
  if (p.rect_w > 0) {
    // rectangle tiles: a plain tiled box per tap; OOB (padding, ragged rects,
    // images past the batch) is zero-filled
    auto enct = get_encode_tiled();
    if (!enct) return nullptr;
    const cuuint32_t box[4] = {(cuuint32_t)(slab / esz), (cuuint32_t)p.rect_w,
                               (cuuint32_t)p.rect_h, (cuuint32_t)p.rect_n};
    const cuuint32_t estr[4] = {1, 1, 1, 1};
    const CUtensorMapSwizzle sw = slab == 128 ? CU_TENSOR_MAP_SWIZZLE_128B
                                  : slab == 64 ? CU_TENSOR_MAP_SWIZZLE_64B
                                               : CU_TENSOR_MAP_SWIZZLE_32B;
    CUresult r = enct(&m, gs.st == ST_BF16 ? CU_TENSOR_MAP_DATA_TYPE_BFLOAT16
                                           : CU_TENSOR_MAP_DATA_TYPE_FLOAT32,
                      4, const_cast<void *>(x), dims, strides, box, estr,
                      CU_TENSOR_MAP_INTERLEAVE_NONE, sw, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                      CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (r != CUDA_SUCCESS) return nullptr;
    if (gs.xmaps.size() > 64) gs.xmaps.clear();
    return &(gs.xmaps[key] = m);
  }
  auto enc = get_encode_im2col();
  if (!enc) return nullptr;
  // bounding box of the conv's input corners (square kernels: W and H equal);
  // a zero-haloed input (perforated variant of a padded-layout layer) is the
  // shared-halo grid [H + ih][W + ih] (interior at the origin): only the
  // extent grows, the traversal box still ends pad - (S - 1) past the interior
  cuuint64_t dimsh[4] = {dims[0], dims[1] + (cuuint64_t)g.ih, dims[2] + (cuuint64_t)g.ih,
                         dims[3]};
  const cuuint64_t stridesh[3] = {(cuuint64_t)g.Cs * esz, dimsh[1] * g.Cs * esz,
                                  dimsh[2] * dimsh[1] * g.Cs * esz};
  const int lower[2] = {-g.pad, -g.pad};
  const int upper[2] = {g.pad - (g.S - 1) - g.ih, g.pad - (g.S - 1) - g.ih};
  const cuuint32_t estr[4] = {1, (cuuint32_t)(g.stride * std::max(g.psw, 1)),
                              (cuuint32_t)(g.stride * std::max(g.psh, 1)), 1};
  const CUtensorMapSwizzle sw = slab == 128 ? CU_TENSOR_MAP_SWIZZLE_128B
                                : slab == 64 ? CU_TENSOR_MAP_SWIZZLE_64B
                                             : CU_TENSOR_MAP_SWIZZLE_32B;
  CUresult r = enc(&m, gs.st == ST_BF16 ? CU_TENSOR_MAP_DATA_TYPE_BFLOAT16
                                        : CU_TENSOR_MAP_DATA_TYPE_FLOAT32,
                   4, const_cast<void *>(x), dimsh, stridesh, lower, upper,
                   (cuuint32_t)(slab / esz), 128, estr, CU_TENSOR_MAP_INTERLEAVE_NONE, sw,
                   CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) return nullptr;
  if (gs.xmaps.size() > 64) gs.xmaps.clear();
  return &(gs.xmaps[key] = m);
}

// Weight map of the weight-streaming FC kernel over the re-tiled layout
// [RB][KB][128][kbe]: a box {kbe, 128, 1, 1} is one contiguous 16 KB tile.
static const CUtensorMap *stage_fcwmap(GemmStage &gs) {
  const int key = -7;
  auto it = gs.tmaps.find(key);
  if (it != gs.tmaps.end()) return &it->second;
  auto enc = get_encode_tiled();
  if (!enc) return nullptr;
  const int esz = esz_of(gs.st), kbe = 128 / esz;
  const cuuint64_t KB = gs.g.Kpad / kbe, RB = (gs.g.Nfg + 127) / 128;
  CUtensorMap m;
  const cuuint64_t dims[4] = {(cuuint64_t)kbe, 128, KB, RB};
  const cuuint64_t strides[3] = {128, 128ull * 128, 128ull * 128 * KB};
  const cuuint32_t box[4] = {(cuuint32_t)kbe, 128, 1, 1};
  const cuuint32_t estr[4] = {1, 1, 1, 1};
  CUresult r = enc(&m, gs.st == ST_BF16 ? CU_TENSOR_MAP_DATA_TYPE_BFLOAT16 : CU_TENSOR_MAP_DATA_TYPE_FLOAT32,
                   4, gs.d_w, dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                   CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                   CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) return nullptr;
  return &(gs.tmaps[key] = m);
}

// Activation (B operand) map of the weight-streaming FC kernel: the input
// [B][K] matrix (K = the stored NHWC flatten), boxes of 128 B of K x nb images,
// SW128; images past the batch and K past the row are zero-filled.
static const CUtensorMap *stage_fcxmap(GemmStage &gs, const void *x, int batch, int nb) {
  const auto key = std::make_tuple(x, batch, nb, -1, -1);
  auto it = gs.xmaps.find(key);
  if (it != gs.xmaps.end()) return &it->second;
  auto enc = get_encode_tiled();
  if (!enc) return nullptr;
  const int esz = esz_of(gs.st);
  CUtensorMap m;
  const cuuint64_t dims[2] = {(cuuint64_t)gs.g.K, (cuuint64_t)batch};
  const cuuint64_t strides[1] = {(cuuint64_t)gs.g.K * esz};
  const cuuint32_t box[2] = {(cuuint32_t)(128 / esz), (cuuint32_t)nb};
  const cuuint32_t estr[2] = {1, 1};
  CUresult r = enc(&m, gs.st == ST_BF16 ? CU_TENSOR_MAP_DATA_TYPE_BFLOAT16 : CU_TENSOR_MAP_DATA_TYPE_FLOAT32,
                   2, const_cast<void *>(x), dims, strides, box, estr,
                   CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
                   CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) return nullptr;
  if (gs.xmaps.size() > 64) gs.xmaps.clear();
  return &(gs.xmaps[key] = m);
}

// Output maps for the epilogue's TMA tensor stores: the [M][out_cs] output
// matrix (rows = output pixels, padded grid in pm mode), boxes of 32 columns
// x 32 rows, swizzle = the box row width (64 B bf16 / 128 B fp32), and for
// bf16 a second map with 64-column boxes (128 B rows, SW128; *y64 = nullptr
// when out_cs < 64).  nullptr when the layout does not meet TMA's alignment
// rules (row stores are used).
static const CUtensorMap *stage_ymap(GemmStage &gs, void *y, long long M,
                                     const CUtensorMap **y64) {
  const ConvGeom &g = gs.g;
  const int eszo = g.out_mode == OUT_BF16 ? 2 : 4;
  *y64 = nullptr;
  if (((uintptr_t)y & 15) || ((long long)g.out_cs * eszo) % 16 || g.out_cs < 32) return nullptr;
  const bool wide = eszo == 2 && g.out_cs >= 64;
  const auto key = std::make_pair((const void *)y, M);
  auto it = gs.ymaps.find(key);
  if (it != gs.ymaps.end()) {
    if (wide) *y64 = &it->second.second;
    return &it->second.first;
  }
  auto enc = get_encode_tiled();
  if (!enc) return nullptr;
  std::pair<CUtensorMap, CUtensorMap> m;
  const cuuint64_t dims[2] = {(cuuint64_t)g.out_cs, (cuuint64_t)M};
  const cuuint64_t strides[1] = {(cuuint64_t)g.out_cs * eszo};
  const cuuint32_t box[2] = {32, 32};
  const cuuint32_t estr[2] = {1, 1};
  CUresult r = enc(&m.first, eszo == 2 ? CU_TENSOR_MAP_DATA_TYPE_BFLOAT16 : CU_TENSOR_MAP_DATA_TYPE_FLOAT32,
                   2, y, dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                   eszo == 2 ? CU_TENSOR_MAP_SWIZZLE_64B : CU_TENSOR_MAP_SWIZZLE_128B,
                   CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) return nullptr;
  m.second = m.first;
  if (wide) {
    const cuuint32_t box64[2] = {64, 32};
    r = enc(&m.second, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, y, dims, strides, box64, estr,
            CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
            CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (r != CUDA_SUCCESS) return nullptr;
  }
  if (gs.ymaps.size() > 64) gs.ymaps.clear();
  auto &slot = gs.ymaps[key] = m;
  if (wide) *y64 = &slot.second;
  return &slot.first;
}

// ------------------------------------------------------------------ planning
// Tile / split selection (the paper's sub-matrix choice, P:223,
// P:267).  For every CTA grouping cg (1 CTA, M = 128 / CTA pair, M = 256) and
// N tile bn (multiple of 32, <= 256):
//   tiles  = ceil(M / (128 cg)) * ceil(Nfg / bn) * groups       (eq. 4)
//   splits = K split when the tiles cannot fill the GPU
//   K-block cost per SM (cycles) = max(MMA ~2.05 bn,
//                                      TMA ~3.6 per 128-B box row x (128 + bn/cg))
//   time   = max(waves * kblocks/splits * cost / f, weight bytes / HBM)
//            + split-K reduction traffic
// (the per-row TMA cost is the measured rate of this kernel on B200; the MMA
// figure is the tcgen05 floor).  Small tiles raise Util (eq. 6) and rEC
// (eq. 9), big tiles raise the computation density per loaded row -- the
// trade-off of P:223.  The plan depends on the problem shape and the device's
// SM count only, never on the SM budget, so every budget runs the same tiles
// and K order (bitwise-identical results, R11).
// Measured on B200 (tools/tc_roles.py, PCNN_TC_SKIP / PCNN_AMODE experiments):
// operand delivery is bound by L2->SM bandwidth (~10 TB/s chip, ~36 B/cycle
// per SM) whether A comes by im2col or by tiled boxes, so one K-block costs
// its operand bytes / 36 B per cycle; rectangle tiles only add padded MMA
// rows and are therefore opt-in (PCNN_AMODE=rect).  The tcgen05 pipe sustains
// ~80% of its nominal rate in this kernel.
static constexpr double kOperandBytesPerCycle = 36.0;
// eq. 12 time-model constants (NEXT-3; fitted, see layer_time_model)
static constexpr double kT0Conv = 14.58, kScaleConv = 0.4985;   // tcgen05 conv: launch us, unit scale
// (profiles/r02_time_model_fit.json; measured with live per-layer events,
// which serialise launches -- inside a CUDA graph with PDL the launch term
// mostly overlaps the previous layer)
static constexpr double kT0Fc = 15.08, kScaleFc = 0.699;   // weight-streaming FC
static constexpr double kT0Simt = 3.0;                     // SIMT kernels (LRN / pool / check path)
static constexpr double kMmaEfficiency = 0.8;

// Best rectangle tile (w x h x n <= 128 output pixels) for rect-mode A loads,
// maximising the fraction of useful MMA rows; {0,0,0} when not applicable.
struct Rect { int w, h, n; double util; };
static Rect best_rect(const ConvGeom &g) {
  Rect best{0, 0, 0, 0.0};
  if (g.stride != 1) return best;
  const long long B = g.M / ((long long)g.Ho * g.Wo);
  const int ws[] = {g.Wo, 8, 16, 32, 64, 128};
  for (int w : ws) {
    if (w < 1 || w > 128 || w > g.Wo) continue;
    for (int h = std::min(128 / w, g.Ho); h >= 1; --h) {
      // FC (1 x 1 "images"): the rectangle spans up to 128 images
      const int n = (g.Ho == 1 && g.Wo == 1) ? (int)std::min<long long>(128, B) : 1;
      const long long rects = ((B + n - 1) / n) * ((g.Ho + h - 1) / h) * ((g.Wo + w - 1) / w);
      const double util = (double)g.M / ((double)rects * 128.0);
      if (util > best.util + 1e-9) best = Rect{w, h, n, util};
    }
  }
  return best;
}

static TcPlan plan_tc(const ConvGeom &g, int device_sms, int kblocks, int esz,
                      bool full_n = false, int want_cg = 0) {
  TcPlan best{};
  double best_t = 1e300;
  const int nmax = std::min(256, round_up(g.Nfg, 32));
  const double f = 1.9e9, hbm = 6.0e12;
  const double wbytes = (double)g.Nfg * g.groups * g.Kpad * esz;
  const char *force_cg = exp_env("PCNN_FORCE_CG");
  const char *force_bn = exp_env("PCNN_FORCE_BN");          // tuning experiments
  const char *force_am = exp_env("PCNN_AMODE");             // "im2col" | "rect"
  if (want_cg > 0) force_cg = want_cg == 1 ? "1" : "2";
  const Rect rc = best_rect(g);
  // Split-K changes an output's summation order.  It is considered only when
  // no tile shape fills the device without it (tiny batches): then the K
  // order of every image is the same for every batch at which some tile
  // shape fills the device -- per-image results are bitwise equal at B and
  // B / W and across pcnn_infer_host's chunks.
  bool can_fill = false;
  for (int cg = 1; cg <= 2; ++cg)
    for (int bn = 32; bn <= std::max(32, nmax); bn += 32) {
      const long long t = ((g.M + 128LL * cg - 1) / (128LL * cg)) * ((g.Nfg + bn - 1) / bn) * g.groups;
      if (t >= device_sms / cg) can_fill = true;
    }
  for (int am = 0; am < 2; ++am) {            // 0 im2col, 1 rectangle tiles (opt-in)
    if (am == 1 && (rc.w == 0 || !force_am || std::string(force_am) != "rect")) continue;
    if (am == 0 && force_am && std::string(force_am) == "rect" && rc.w != 0) continue;
    const long long rows_total = am ? (long long)std::llround(g.M / rc.util) : g.M;
    const double a_bytes = 128.0 * (am ? rc.w * rc.h * rc.n : 128);
    for (int cg = 1; cg <= 2; ++cg) {
      if (force_cg && atoi(force_cg) != cg) continue;
      const int mtiles = (int)((rows_total + 128LL * cg - 1) / (128LL * cg));
      const int slots = device_sms / cg;          // concurrent units
      for (int bn = 32; bn <= std::max(32, nmax); bn += 32) {   // epilogue drains 32 columns
        if (full_n && bn != round_up(g.Nfg, 32)) continue;      // one N tile (fused LRN)
        if (force_bn && !full_n && atoi(force_bn) != bn) continue;
        const int ntiles = (g.Nfg + bn - 1) / bn;
        const long long tiles = (long long)mtiles * ntiles * g.groups;
        const double load = (a_bytes + 128.0 * bn / cg) / kOperandBytesPerCycle;
        const double mma = 2.05 * bn / kMmaEfficiency;
        const double kb_cycles = std::max(load, mma) + 40.0;
        // split-K candidates: none, or any split that keeps >= 4 K-blocks per unit
        const int max_split =
            (tiles >= slots || full_n || can_fill) ? 1 : std::min(16, std::max(1, kblocks / 4));
        static const int force_split = [] {              // tuning experiments
          const char *e = exp_env("PCNN_FORCE_SPLIT");
          return e ? atoi(e) : 0;
        }();
        for (int want = 1; want <= max_split; ++want) {
          const int kbs = (kblocks + want - 1) / want;
          const int splits = (kblocks + kbs - 1) / kbs;
          if (splits != want) continue;
          if (force_split > 0 && splits != force_split) continue;
          const long long units = tiles * splits;
          const long long waves = (units + slots - 1) / slots;
          double t = (double)waves * kbs * kb_cycles / f + 2e-6;   // + per-tile drain
          t = std::max(t, wbytes / hbm);
          if (splits > 1) t += (double)g.M * g.Nfg * g.groups * 4.0 * (splits + 1) / hbm + 3e-6;
          if (t < best_t * 0.999 ||
              (t <= best_t * 1.001 && (long long)bn * cg > (long long)best.bn * best.cg)) {
            best_t = t;
            best.cg = cg;
            best.bn = bn;
            best.mtiles = mtiles;
            best.ntiles = ntiles;
            best.tiles = (int)tiles;
            best.splits = splits;
            best.kb_per_split = kbs;
            best.units = (int)units;
            best.unit_us = ((double)kbs * kb_cycles / f + 2e-6) * 1e6;
            best.rect_w = am ? rc.w : 0;
            best.rect_h = am ? rc.h : 0;
            best.rect_n = am ? rc.n : 0;
          }
        }
      }
    }
  }
  return best;
}

// Padded-layout plan: per (slab, filter row) window the SM loads
// (128 + S - 1) A rows once plus S weight slabs and issues S x slab/32 UMMAs;
// no split-K (a split would need the halo zeroing in the reduction).
static TcPlan plan_tc_pm(const ConvGeom &g, int device_sms, int esz, bool full_n = false,
                         int want_cg = 0, int want_msub = 0, bool per_row = false) {
  TcPlan best{};
  double best_t = 1e300;
  std::vector<std::pair<double, TcPlan>> cands;
  const int nmax = std::min(256, round_up(g.Nfg, 32));
  const double f = 1.9e9;
  const int slab = tc_slab_bytes(esz == 2 ? ST_BF16 : ST_F32, g.Cg);
  const int nj = g.Cg * esz / slab * g.S;
  const char *force_cg = exp_env("PCNN_FORCE_CG");
  const char *force_bn = exp_env("PCNN_FORCE_BN");
  const char *force_ms = exp_env("PCNN_PM_MSUB");           // 1 | 2 (experiments)
  if (want_cg > 0) force_cg = want_cg == 1 ? "1" : "2";
  if (want_msub > 0) force_ms = want_msub == 1 ? "1" : "2";
  // split-K over the windows only when no tile shape fills the device (tiny
  // batches; R17: the K order of an image is then batch-independent for every
  // batch at which some tile shape fills it); row perforation (pm = 2) never
  bool can_fill = false;
  for (int ms = 1; ms <= 2; ++ms)
    for (int cg = 1; cg <= 2; ++cg)
      for (int bn = 32; bn <= std::max(32, nmax); bn += 32) {
        if (ms == 2 && bn > 128) continue;
        const long long t = ((g.M + 128LL * cg * ms - 1) / (128LL * cg * ms)) *
                            ((g.Nfg + bn - 1) / bn) * g.groups;
        if (t >= device_sms / cg) can_fill = true;
      }
  // Measured (tools/exp_b1_split.sh, AlexNet B = 1, graph replay): the
  // split-K plans' partial epilogues and reduction launches cost more than the
  // extra CTAs gain (0.124 vs 0.1205 ms per pass), so padded-layout plans do
  // not split K; the experiments build can still force a split.
  static const int force_split = [] {              // tuning experiments
    const char *e = exp_env("PCNN_FORCE_SPLIT");
    return e ? atoi(e) : 0;
  }();
  const int max_split =
      (can_fill || full_n || g.pm != 1 || force_split <= 1) ? 1 : std::min(16, nj);
  static const int force_ww = [] {                 // A/B experiments: 0 off, 1 forced
    const char *e = exp_env("PCNN_WW");
    return e ? atoi(e) : -1;
  }();
  const double hbm = 6.0e12;
  for (int ms = 1; ms <= 2; ++ms) {
    if (force_ms && atoi(force_ms) != ms) continue;
    for (int cg = 1; cg <= 2; ++cg) {
      if (force_cg && atoi(force_cg) != cg) continue;
      const long long rows = 128LL * cg * ms;
      const int mtiles = (int)(((long long)g.M + rows - 1) / rows);
      const int slots = device_sms / cg;
      for (int bn = 32; bn <= std::max(32, nmax); bn += 32) {
        if (full_n && bn != round_up(g.Nfg, 32)) continue;     // one N tile (fused LRN)
        if (force_bn && !full_n && atoi(force_bn) != bn) continue;
        if (ms == 2 && bn > 128) continue;          // two accumulators per TMEM buffer
        const int ntiles = (g.Nfg + bn - 1) / bn;
        const long long tiles = (long long)mtiles * ntiles * g.groups;
        // per (slab, filter row): ms windows of 128 + S - 1 rows and S weight
        // slabs (shared by the ms sub-tiles) through L2, each TMA load with a
        // fixed issue / completion cost (measured: ~64 cycles; AlexNet conv2
        // ms = 1 1970 cycles per window vs 1680 from bytes and MMAs alone),
        // ms * S UMMA slabs of which the last channel slab's zero padding is
        // skipped (kmma_eff of slab/32 UMMAs, averaged over the slabs)
        const int se = slab / esz, ncb = std::max(1, g.Cg / se);
        const int creal = g.Creal > 0 && g.Creal <= g.Cg ? g.Creal : g.Cg;
        const double last_frac =
            std::min(1.0, std::ceil((double)(creal - (ncb - 1) * se) * esz / 32.0) / (slab / 32.0));
        const double kfrac = ((ncb - 1) + last_frac) / ncb;
        // whole windows (ww = 1, no split-K): one A window of 128 + (S-1)(wv+1)
        // rows per channel slab feeds all S x S taps, instead of S windows of
        // 128 + S - 1 rows (one per filter row) -- fewer A bytes when wv is
        // small against 128 (AlexNet conv1-5, VGG-16 conv2-5)
        for (int ww = 0; ww <= 1; ++ww) {
          if (ww && (per_row || g.pm != 1 || pm_window_rows(g.S, g.wv, 1) > 256 || g.S < 2 ||
                     pm_window_rows(g.S, g.wv, 1) >= g.S * (128 + g.S - 1) || force_ww == 0))
            continue;
          if (!ww && force_ww == 1 && g.pm == 1 && pm_window_rows(g.S, g.wv, 1) <= 256) continue;
          const int rows = pm_window_rows(g.S, g.wv, ww);
          const int taps = ww ? g.S * g.S : g.S, nwin = ww ? nj / g.S : nj;
          {   // the A ring must hold 2 windows next to 8 tap slabs
            int na = 0, nb = 0;
            tc_pm_stages(bn, cg, slab, g.S, ms, &na, &nb, rows, ww);
            if (na < 2 || nb < (ww ? 6 : 2)) continue;
          }
          const double load = (ms * (double)rows * slab + (double)taps * slab * bn / cg) /
                                  kOperandBytesPerCycle + 64.0 * (ms + taps);
          const double mma = ms * taps * (slab / 128.0) * kfrac * 2.05 * bn / kMmaEfficiency;
          // + the issuer's per-tap cost (full-barrier wait, fence, commit; ~100
          // cycles measured: without it narrow-N whole-window plans, e.g.
          // AlexNet conv4 512 x 64, model faster than the 256 x 192 that wins)
          const double j_cycles = std::max(load, mma) + 40.0 + 100.0 * taps;
          for (int want = 1; want <= (ww ? 1 : max_split); ++want) {
            const int kbs = (nwin + want - 1) / want;
            const int splits = (nwin + kbs - 1) / kbs;
            if (splits != want) continue;
            if (force_split > 0 && splits != force_split && max_split >= force_split) continue;
            const long long units = tiles * splits;
            const long long waves = (units + slots - 1) / slots;
            double t = (double)waves * kbs * j_cycles / f + 2e-6 * ms;
            // partials written and summed by the reduction launch
            if (splits > 1) t += (double)g.M * g.Nfg * g.groups * 4.0 * (splits + 1) / hbm + 3e-6;
            TcPlan c{};
            c.cg = cg;
            c.bn = bn;
            c.msub = ms;
            c.ww = ww;
            c.mtiles = mtiles;
            c.ntiles = ntiles;
            c.tiles = (int)tiles;
            c.splits = splits;
            c.kb_per_split = kbs;
            c.units = (int)units;
            c.unit_us = ((double)kbs * j_cycles / f + 2e-6 * ms) * 1e6;
            cands.push_back({t, c});
            best_t = std::min(best_t, t);
          }
        }
      }
    }
  }
  // within 5% of the fastest modelled plan (the model's error on measured
  // layers), prefer the widest N tile: it re-reads A the fewest times (VGG
  // conv3-5: 256 x 256 beats 512 x 128 by ~4% although modelled 2% slower)
  long long wide = -1;
  double bt = 1e300;
  for (auto &pc : cands) {
    if (pc.first > best_t * 1.05) continue;
    const long long wdt = (long long)pc.second.bn * pc.second.cg;
    if (wdt > wide || (wdt == wide && pc.first < bt)) {
      wide = wdt;
      bt = pc.first;
      best = pc.second;
    }
  }
  tc_pm_stages(best.bn, best.cg, slab, g.S, best.msub, &best.a_stages, &best.b_stages,
               pm_window_rows(g.S, g.wv, best.ww), best.ww);
  return best;
}

// Weight-streaming FC plan (kernels_fc.cu).  The K split s (CTA pairs per
// 256-row unit) and its ranges come from the layer shape and the device's SM
// count only -- never from the batch or the SM budget -- so every image's sum
// runs in the same order for any batch (bitwise per-image results at B and
// B / W) and any budget (R11).  s is the largest power
// of two <= 16 that keeps >= 4 K-blocks per split and fits all row blocks'
// pairs on the device at once.  The batch only picks the UMMA N (nb images
// per chunk) and the number of chunks, which move work between CTA pairs but
// never change a sum.  All CTAs of the launch must be co-resident (the
// split-K partials meet at a global counter): grid <= SM budget, and a budget
// below 2 s SMs is raised to 2 s.
static FcPlan plan_fc(int N, int kblocks, int B, int device_sms, int budget_sms) {
  FcPlan p{};
  const int rb = (N + 255) / 256;
  int s = 1;
  while (s < 16 && rb * 2 * (2 * s) <= device_sms && kblocks / (2 * s) >= 4) s *= 2;
  // (the kernel gives split j the K-blocks [j KB / s, (j + 1) KB / s): never empty)
  if (const char *e = exp_env("PCNN_FC_SPLIT")) s = atoi(e);   // experiments build only
  p.splits = s;
  p.kbps = (kblocks + s - 1) / s;
  p.chunks = (B + 255) / 256;
  p.nb = round_up((B + p.chunks - 1) / p.chunks, 16);
  p.rblocks = rb;
  const int units = p.rblocks * p.chunks;
  p.groups = std::max(1, std::min(units, std::min(budget_sms, device_sms) / (2 * s)));
  p.grid = 2 * s * p.groups;
  // per K-block a CTA ingests one contiguous 16 KB weight tile + nb / 2
  // activation rows at the measured ~60 B/clk/SM of this kernel's TMA stream
  // (tools/time_model_fit.py: 5.4 us per 590 KB unit of fc6 at batch 1); the
  // pair's MMA (256 x nb x 64) takes nb / 2 cycles per 16-deep UMMA step x 4
  const double f = 1.9e9;
  const double load = (16384.0 + 64.0 * p.nb) / 60.0, mma = 4.0 * std::max(16, p.nb / 2) / 0.8;
  // + the split-K partial tile (written, then s slices of it read back by
  // the reduction): 2 x 128 rows x nb x 4 B per CTA through L2
  const double red = s > 1 ? 2.0 * 128.0 * p.nb * 4.0 / 36.0 : 0.0;
  p.unit_us = ((double)p.kbps * (std::max(load, mma) + 40.0) / f + red / f + 2e-6) * 1e6;
  return p;
}

static int effective_sms(const pcnn_net *net, const Layer &ly) {
  int n = ly.n_sms <= 0 ? net->num_sms : std::min(ly.n_sms, net->num_sms);
  return std::max(n, 1);
}

static bool is_gated(const pcnn_net *net, const Layer &ly) {
  return (ly.n_sms > 0 && ly.n_sms < net->num_sms) || ly.tlp > 0;
}

static Budget make_budget(const pcnn_net *net, const Layer &ly, int slot, bool gated_kernel) {
  Budget b{};
  b.gated = gated_kernel && is_gated(net, ly) ? 1 : 0;
  b.n_sms = effective_sms(net, ly);
  b.tlp = ly.tlp > 0 ? ly.tlp : 1 << 20;
  b.ctr = ly.d_ctr + (size_t)slot * (1 + kMaxSMs);
  b.census = net->census ? ly.d_census : nullptr;
  return b;
}

// ------------------------------------------------------------------ enqueue
static pcnn_status run_stage(pcnn_net *net, Layer &ly, GemmStage &gs, int B, const void *x,
                             void *y, int slot, cudaStream_t s, pcnn_layer_info *info,
                             size_t *ws_need = nullptr, const float *lrn = nullptr) {
  ConvGeom g = gs.g;
  g.M = g.pm == 2 ? B * g.tpi * 128 : g.pm ? B * g.hv * g.wv : B * g.Ho * g.Wo;
  if (gs.engine == 1 && gs.is_fc && !lrn) {
    // a6: weight-streaming FC kernel
    const int N = g.Nfg, kblocks = g.Kpad / tc_block_k_elems(gs.st);
    const FcPlan p = plan_fc(N, kblocks, B, net->num_sms, effective_sms(net, ly));
    if (info) {
      info->tile_m = 256;
      info->tile_n = p.nb;
      info->tiles = (long long)p.rblocks * p.chunks;
      info->grid = p.grid;
      info->tlp = 1;
      info->engine = 1;
      info->splits = p.splits;
      info->a_mode = 3;
      info->n_sms = std::max(info->n_sms, p.grid);
      info->cta_group = 2;
      info->t_unit_us = p.unit_us;
    }
    const size_t wsb = p.splits > 1 ? (size_t)p.splits * B * N * 4 : 0;
    if (ws_need) *ws_need = std::max(*ws_need, wsb);
    const int units = p.rblocks * p.chunks;
    if (ws_need && 2 * units > gs.sem_count) {
      // split-K arrival counters (reserved with the workspace, outside any
      // graph capture): zeroed once, re-armed by the kernel itself
      CUDA_TRY(cudaDeviceSynchronize());
      if (gs.d_sem) cudaFree(gs.d_sem);
      gs.d_sem = nullptr;
      gs.sem_count = 0;
      CUDA_TRY(cudaMalloc(&gs.d_sem, sizeof(unsigned) * 2 * units));
      CUDA_TRY(cudaMemset(gs.d_sem, 0, sizeof(unsigned) * 2 * units));
      gs.sem_count = 2 * units;
      net->version++;          // cached graphs captured the old pointer
    }
    if (!x) return PCNN_OK;
    if (wsb > net->ws_bytes) return fail(PCNN_ERR_OUT_OF_MEMORY, "FC split-K workspace not reserved");
    if (p.splits > 1 && 2 * units > gs.sem_count)
      return fail(PCNN_ERR_OUT_OF_MEMORY, "FC split-K counters not reserved");
    const CUtensorMap *tm = stage_fcwmap(gs);
    const CUtensorMap *xm = stage_fcxmap(gs, x, B, p.nb / 2);
    if (!tm || !xm) return fail(PCNN_ERR_CUDA, "cuTensorMapEncodeTiled failed (FC)");
    Budget b = make_budget(net, ly, slot, false);
    CUDA_TRY(counted(launch_fc_tc(p, gs.st, tm, xm, gs.d_bias, y, net->d_ws, gs.d_sem, N, B,
                                  kblocks, g.relu, g.out_mode, g.out_cs, b, s)));
    return PCNN_OK;
  }
  if (gs.engine == 1) {
    TcPlan p = g.pm ? plan_tc_pm(g, net->num_sms, esz_of(gs.st), lrn != nullptr, ly.plan_cg,
                                 ly.plan_msub, net->per_row_windows)
                    : plan_tc(g, net->num_sms, g.Kpad / tc_block_k_elems(gs.st), esz_of(gs.st),
                              lrn != nullptr, ly.plan_cg);
    // the budget caps concurrent units; a CTA pair needs at least 2 SMs
    const int slots = std::max(1, effective_sms(net, ly) / p.cg);
    p.grid = p.cg * std::min(p.units, slots);
    // weight rows per CTA; padded mode loads one tap's slab per stage
    const CUtensorMap *tm =
        stage_tmap(gs, p.bn / p.cg, g.pm ? tc_slab_bytes(gs.st, g.Cg) : 128);
    if (!tm) return fail(PCNN_ERR_CUDA, "cuTensorMapEncodeTiled failed");
    if (info) {
      info->tile_m = 128 * p.cg * std::max(1, p.msub);
      info->tile_n = p.bn;
      info->tiles = p.tiles;
      info->grid = p.grid;
      info->tlp = 1;
      info->engine = 1;
      info->splits = p.splits;
      info->a_mode = g.pm ? 2 : (p.rect_w ? 1 : 0);
      info->whole_window = p.ww;
      info->n_sms = std::max(info->n_sms, p.grid);   // pair granularity
      info->cta_group = p.cg;
      info->t_unit_us = p.unit_us;
    }
    if (ws_need) *ws_need = std::max(*ws_need, p.splits > 1 ? (size_t)p.splits * g.M * g.out_cs * 4 : 0);
    if (!x) return PCNN_OK;   // planning only
    const CUtensorMap *xm = stage_xmap(gs, x, B, p);
    if (!xm) return fail(PCNN_ERR_CUDA, "cuTensorMapEncodeIm2col failed");
    Budget b = make_budget(net, ly, slot, false);
    if (p.splits > 1 && (size_t)p.splits * g.M * g.out_cs * 4 > net->ws_bytes)
      return fail(PCNN_ERR_OUT_OF_MEMORY, "split-K workspace not reserved");
    g_launches += p.splits > 1 ? 1 : 0;   // the reduction kernel
    static const bool no_tma_store = [] {
      const char *e = exp_env("PCNN_NO_TMA_STORE");
      return e && e[0] == '1';
    }();
    static const bool no_wide = [] {
      const char *e = exp_env("PCNN_NO_WIDE_STORE");
      return e && e[0] == '1';
    }();
    const CUtensorMap *ym64 = nullptr;
    const CUtensorMap *ym = (p.splits == 1 && !lrn && !p.rect_w && !no_tma_store && g.pm != 2)
                                ? stage_ymap(gs, y, g.M, &ym64) : nullptr;
    if (no_wide) ym64 = nullptr;
    CUDA_TRY(counted(launch_conv_tc(g, gs.st, xm, tm, gs.d_bias, y, gs.d_ktab, p, net->d_ws,
                                    b, s, lrn, ym, ym64)));
  } else {
    const int tiles = conv_simt_tiles(g);
    const bool gated = is_gated(net, ly);
    int grid = gated ? net->num_sms * net->occ_simt : tiles;
    if (!gated) grid = std::min(grid, 1 << 30);
    if (info) {
      int tm, tn;
      conv_simt_tile_shape(&tm, &tn);
      info->tile_m = tm;
      info->tile_n = tn;
      info->tiles = tiles;
      info->grid = grid;
      info->tlp = ly.tlp > 0 ? ly.tlp : net->occ_simt;
      info->engine = 0;
      info->cta_group = 1;
      // one tm x tn tile over K at ~60% of 128 FFMA lanes, occ_simt CTAs per SM
      info->t_unit_us = 2.0 * tm * tn * g.K / (0.6 * 256.0 * 1.9e9) * 1e6 * net->occ_simt;
    }
    if (!x) return PCNN_OK;
    Budget b = make_budget(net, ly, slot, true);
    if (b.gated)
      CUDA_TRY(cudaMemsetAsync(b.ctr, 0, sizeof(unsigned long long) * (1 + kMaxSMs), s));
    CUDA_TRY(counted(launch_conv_simt(g, (const float *)x, (const float *)gs.d_w, gs.d_bias,
                              (float *)y, gs.d_ktab, b, grid, s)));
  }
  return PCNN_OK;
}

// conv layer i immediately followed by a size-5 LRN that the conv epilogue can
// apply in registers: tcgen05 engine, exact variant, one group, every output
// channel in one N tile (<= 128).
static bool fuse_conv_lrn(const pcnn_net *net, int i) {
  if (!net->fuse_lrn_pool || i + 1 >= (int)net->layers.size()) return false;
  const Layer &c = net->layers[i], &l = net->layers[i + 1];
  // padded-layout convs fuse LRN only on request (PCNN_FLAG_CONV_LRN_EPILOGUE):
  // even the 8-warp streaming LRN epilogue makes AlexNet conv1 161 us (+ 49 us
  // for the then stand-alone pool1) against 84 us conv + 90 us LRN+pool kernel
  // at B = 256: two epilogue warps per SM sub-partition cannot hide the
  // per-element MUFU work (round 1's 4-warp epilogue: 279 us)
  const bool pm_lrn = net->conv_lrn_pm;
  return c.d.kind == PCNN_CONV && l.d.kind == PCNN_LRN && l.d.kernel == 5 &&
         (c.pm_halo == 0 || pm_lrn) && c.perf_sh * c.perf_sw == 1 &&
         c.exact.engine == 1 && c.variant == PCNN_VARIANT_EXACT && c.d.groups == 1 &&
         c.d.out_channels <= 128 && c.out_cs == c.d.out_channels;
}

static void lrn_params(const Layer &l, float p[4]) {
  p[0] = (float)l.d.kernel;
  p[1] = l.d.lrn_alpha;
  p[2] = l.d.lrn_beta;
  p[3] = l.d.lrn_k;
}

// LRN layer `li` and / or pooling layer `pi` (-1 = absent) in one launch
// (the fused pair runs under the LRN layer's budget).
static pcnn_status run_lrn_pool(pcnn_net *net, int li, int pi, int B, const void *x, void *y,
                                cudaStream_t s) {
  Layer &ly = net->layers[li >= 0 ? li : pi];
  const int C = ly.in_cs, H = ly.in_h, W = ly.in_w;
  int lrn = 0, k = 1, st = 1, is_max = 1, Ho = H, Wo = W;
  float alpha = 0.f, beta = 0.f, kk = 1.f;
  if (li >= 0) {
    const auto &d = net->layers[li].d;
    lrn = d.kernel;
    alpha = d.lrn_alpha;
    beta = d.lrn_beta;
    kk = d.lrn_k;
  }
  if (pi >= 0) {
    const Layer &p = net->layers[pi];
    k = p.d.kernel;
    st = p.d.stride;
    is_max = p.d.kind == PCNN_MAXPOOL;
    Ho = p.out_h;
    Wo = p.out_w;
  }
  const long long tiles = lrn_pool_tiles(net->st, B, W, C, lrn, k, st, Ho, Wo);
  const bool gated = is_gated(net, ly);
  const int grid = gated ? net->num_sms * net->occ_lp : (int)std::min<long long>(tiles, 1 << 30);
  Budget b = make_budget(net, ly, 0, true);
  if (b.gated)
    CUDA_TRY(cudaMemsetAsync(b.ctr, 0, sizeof(unsigned long long) * (1 + kMaxSMs), s));
  const Layer &last = net->layers[pi >= 0 ? pi : li];
  CUDA_TRY(counted(launch_lrn_pool(x, y, net->st, net->desc.precision == PCNN_TF32, B, H, W, C,
                                   lrn, alpha, beta, kk, k, st, is_max, Ho, Wo, last.out_groups,
                                   last.out_cg_pad, ly.in_halo, last.out_halo, b, grid, s)));
  return PCNN_OK;
}

// Enqueue one layer.  x / y are arena buffers (or the user's output for a
// final FC).  r_buf is the rank-r intermediate buffer.
static pcnn_status run_layer(pcnn_net *net, int i, int B, const void *x, void *y, void *r_buf,
                             cudaStream_t s) {
  Layer &ly = net->layers[i];
  const int st = net->st;
  const int tf32 = net->desc.precision == PCNN_TF32;
  switch (ly.d.kind) {
    case PCNN_CONV:
    case PCNN_FC:
      if (ly.perf_sh * ly.perf_sw > 1 && ly.pf.g.pm == 2) {
        // row perforation in padded-layout mode: the epilogue writes each
        // kept row to every output row it stands for (R13); the halo rows
        // above / below the image are zeroed here
        pcnn_status r = run_stage(net, ly, ly.pf, B, x, y, 0, s, nullptr);
        if (r != PCNN_OK) return r;
        const ConvGeom &g = ly.pf.g;
        const size_t rowb = (size_t)g.wv * ly.out_cs * esz_of(ly.pf.st);
        const size_t img = (size_t)g.hv * rowb;
        if (g.vh > 0) CUDA_TRY(cudaMemset2DAsync(y, img, 0, (size_t)g.vh * rowb, B, s));
        CUDA_TRY(cudaMemset2DAsync((char *)y + (size_t)(g.vh + g.Ho) * rowb, img, 0,
                                   (size_t)(g.hv - g.vh - g.Ho) * rowb, B, s));
        return PCNN_OK;
      }
      if (ly.perf_sh * ly.perf_sw > 1) {
        // perforation: the conv at the kept grid into the scratch buffer, then
        // nearest-neighbour interpolation into the layer's output layout
        pcnn_status r = run_stage(net, ly, ly.pf, B, x, r_buf, 0, s, nullptr);
        if (r != PCNN_OK) return r;
        CUDA_TRY(counted(launch_perf_interp(r_buf, y, st, B, ly.out_h, ly.out_w, ly.perf_sh,
                                            ly.perf_sw, ly.out_cs, ly.out_halo, s)));
        return PCNN_OK;
      }
      if (ly.variant == PCNN_VARIANT_RANK) {
        pcnn_status r = run_stage(net, ly, ly.r1, B, x, r_buf, 0, s, nullptr);
        if (r != PCNN_OK) return r;
        return run_stage(net, ly, ly.r2, B, r_buf, y, 1, s, nullptr);
      }
      return run_stage(net, ly, ly.exact, B, x, y, 0, s, nullptr);
    case PCNN_LRN:
      return run_lrn_pool(net, i, -1, B, x, y, s);
    case PCNN_MAXPOOL:
    case PCNN_AVGPOOL:
      return run_lrn_pool(net, -1, i, B, x, y, s);
  }
  return fail(PCNN_ERR_INVALID_ARGUMENT, "bad layer kind");
}

static bool last_is_fc(const pcnn_net *net) { return net->layers.back().d.kind == PCNN_FC; }

// The full pass: staging, every layer, unstaging, softmax + entropy.
static pcnn_status enqueue_all(pcnn_net *net, const float *d_images, int B, float *d_out,
                               float *d_p, float *d_h, cudaStream_t s,
                               std::vector<cudaEvent_t> *evs) {
  const int st = net->st;
  const int tf32 = net->desc.precision == PCNN_TF32;
  g_launches = 0;
  if (net->census)
    for (auto &ly : net->layers) CUDA_TRY(cudaMemsetAsync(ly.d_census, 0, 32, s));
  if (net->stage_im2col) {
    const Layer &l0 = net->layers[0];
    CUDA_TRY(counted(launch_stage_im2col(d_images, net->d_act[0], st, B, net->desc.in_channels,
                                         net->desc.in_height, net->desc.in_width, l0.d.kernel,
                                         l0.d.stride, l0.d.pad, l0.out_h, l0.out_w, net->in_cs,
                                         l0.in_halo, tf32, s)));
  } else {
    CUDA_TRY(counted(launch_stage_input(d_images, net->d_act[0], st, B, net->desc.in_channels,
                                        net->desc.in_height, net->desc.in_width, net->stage_h,
                                        net->stage_w, net->in_cs, net->stage_blk,
                                        net->stage_pad, tf32, s)));
  }
  if (evs) CUDA_TRY(cudaEventRecord((*evs)[0], s));
  int cur = 0;
  const int n = (int)net->layers.size();
  for (int i = 0; i < n; ++i) {
    const bool final_fc = (i == n - 1) && last_is_fc(net);
    void *dst = final_fc ? (void *)d_out : net->d_act[cur ^ 1];
    if (fuse_conv_lrn(net, i)) {          // conv + LRN in one launch
      float lp[4];
      lrn_params(net->layers[i + 1], lp);
      Layer &ly = net->layers[i];
      pcnn_status r = run_stage(net, ly, ly.exact, B, net->d_act[cur], dst, 0, s, nullptr,
                                nullptr, lp);
      if (r != PCNN_OK) return r;
      if (evs) {
        CUDA_TRY(cudaEventRecord((*evs)[i + 1], s));
        CUDA_TRY(cudaEventRecord((*evs)[i + 2], s));
      }
      cur ^= 1;
      ++i;
      continue;
    }
    if (net->fuse_lrn_pool && net->layers[i].d.kind == PCNN_LRN && i + 1 < n &&
        (net->layers[i + 1].d.kind == PCNN_MAXPOOL || net->layers[i + 1].d.kind == PCNN_AVGPOOL)) {
      pcnn_status r = run_lrn_pool(net, i, i + 1, B, net->d_act[cur], dst, s);
      if (r != PCNN_OK) return r;
      if (evs) {
        CUDA_TRY(cudaEventRecord((*evs)[i + 1], s));
        CUDA_TRY(cudaEventRecord((*evs)[i + 2], s));
      }
      cur ^= 1;
      ++i;
      continue;
    }
    pcnn_status r = run_layer(net, i, B, net->d_act[cur], dst, net->d_act[2], s);
    if (r != PCNN_OK) return r;
    if (evs) CUDA_TRY(cudaEventRecord((*evs)[i + 1], s));
    if (!final_fc) cur ^= 1;
  }
  if (!last_is_fc(net)) {
    const Layer &l = net->layers.back();
    CUDA_TRY(counted(launch_unstage_output(net->d_act[cur], st, d_out, B, l.out_c, l.out_h, l.out_w,
                                   l.out_cs, s)));
  }
  if (d_p || d_h) CUDA_TRY(counted(launch_softmax_entropy(d_out, d_p, d_h, B, net->out_elems, s)));
  net->launches_per_infer = g_launches;
  return PCNN_OK;
}

// ------------------------------------------------------------------ rank-r
static pcnn_status build_rank_stages(pcnn_net *net, Layer &ly, int r, const float *A,
                                     const float *Bf) {
  // A: [g][Nfg][r], Bf: [g][r][Cg][S][S]
  const auto &d = ly.d;
  const int g = d.groups, Nfg = d.out_channels / g, Cg = ly.in_c / g, S = d.kernel;
  const int prec = net->desc.precision;
  const int st = net->st;
  const int ch = chunk_elems(prec);
  // stage-1 output channels: g*r stored as groups of r; keep each group's r
  // chunk-aligned for the stage-2 gather (pad r with zero filters).
  const int rs = round_up(r, ch);
  std::vector<float> w1((size_t)g * rs * Cg * S * S, 0.f);
  for (int gi = 0; gi < g; ++gi)
    for (int a = 0; a < r; ++a)
      std::memcpy(&w1[((size_t)gi * rs + a) * Cg * S * S], &Bf[((size_t)gi * r + a) * Cg * S * S],
                  sizeof(float) * Cg * S * S);
  std::vector<float> w2((size_t)g * Nfg * rs, 0.f);   // [g*Nfg][rs][1][1]
  for (int gi = 0; gi < g; ++gi)
    for (int f = 0; f < Nfg; ++f)
      for (int a = 0; a < r; ++a)
        w2[((size_t)gi * Nfg + f) * rs + a] = A[((size_t)gi * Nfg + f) * r + a];
  const int mode1 = st == ST_BF16 ? OUT_BF16 : (prec == PCNN_TF32 ? OUT_F32_TF32 : OUT_F32);
  // a padded-layout layer keeps its halo grid through both stages
  pcnn_status s1 = build_stage(ly.r1, ly, prec, g * rs, g, S, d.stride, d.pad, 0, ly.in_c,
                               ly.in_h, ly.in_w, ly.in_cs, false, w1.data(), nullptr, mode1,
                               ly.pm_halo);
  if (s1 != PCNN_OK) return s1;
  const int ho = ly.out_h, wo = ly.out_w;
  const GemmStage &ex = ly.exact;
  pcnn_status s2 = build_stage(ly.r2, ly, prec, d.out_channels, g, 1, 1, 0, d.relu, g * rs, ho,
                               wo, g * rs, false, w2.data(), nullptr, ex.g.out_mode, ly.pm_halo);
  if (s2 != PCNN_OK) return s2;
  // stage 2 carries the layer's bias: copy it from the exact stage.
  CUDA_TRY(cudaMemcpy(ly.r2.d_bias, ex.d_bias, sizeof(float) * d.out_channels,
                      cudaMemcpyDeviceToDevice));
  ly.rank = r;
  ly.variant = PCNN_VARIANT_RANK;
  net->version++;
  return PCNN_OK;
}

// Reserve the split-K workspace for `batch` (outside any graph capture).
static pcnn_status ensure_workspace(pcnn_net *net, int batch) {
  size_t need = 0;
  for (auto &ly : net->layers) {
    if (!ly.gemm) continue;
    if (ly.perf_sh * ly.perf_sw > 1) {
      run_stage(net, ly, ly.pf, batch, nullptr, nullptr, 0, nullptr, nullptr, &need);
    } else if (ly.variant == PCNN_VARIANT_RANK) {
      run_stage(net, ly, ly.r1, batch, nullptr, nullptr, 0, nullptr, nullptr, &need);
      run_stage(net, ly, ly.r2, batch, nullptr, nullptr, 0, nullptr, nullptr, &need);
    } else {
      run_stage(net, ly, ly.exact, batch, nullptr, nullptr, 0, nullptr, nullptr, &need);
    }
  }
  if (need <= net->ws_bytes) return PCNN_OK;
  if (net->d_ws) {
    CUDA_TRY(cudaDeviceSynchronize());
    cudaFree(net->d_ws);
    net->d_ws = nullptr;
    net->ws_bytes = 0;
  }
  if (cudaMalloc(&net->d_ws, need) != cudaSuccess) {
    cudaGetLastError();
    return fail(PCNN_ERR_OUT_OF_MEMORY, "split-K workspace");
  }
  net->ws_bytes = need;
  net->version++;          // cached graphs captured the old pointer
  return PCNN_OK;
}

// ------------------------------------------------------------------ C ABI
extern "C" {

const char *pcnn_version(void) { return "pcnn-b200 0.1 (sm_100a)"; }

const char *pcnn_status_string(pcnn_status s) {
  switch (s) {
    case PCNN_OK: return "ok";
    case PCNN_ERR_INVALID_ARGUMENT: return "invalid argument";
    case PCNN_ERR_SHAPE: return "shape error";
    case PCNN_ERR_UNSUPPORTED: return "unsupported";
    case PCNN_ERR_OUT_OF_MEMORY: return "out of memory";
    case PCNN_ERR_CUDA: return "CUDA error";
    case PCNN_ERR_BATCH_TOO_LARGE: return "batch too large";
  }
  return "unknown status";
}

const char *pcnn_last_error_message(void) { return g_err.c_str(); }

int pcnn_device_sm_count(int device) {
  int n = 0;
  if (cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, device) != cudaSuccess) {
    cudaGetLastError();
    return 0;
  }
  return n;
}

pcnn_status pcnn_describe_net(const pcnn_net_desc *desc, const pcnn_layer_desc *layers,
                              int n_layers, int batch, pcnn_layer_info *infos) {
  if (!infos || batch <= 0) return fail(PCNN_ERR_INVALID_ARGUMENT, "null infos / bad batch");
  std::vector<Layer> ls;
  pcnn_status s = infer_shapes(desc, layers, n_layers, ls);
  if (s != PCNN_OK) return s;
  for (int i = 0; i < n_layers; ++i) {
    const Layer &ly = ls[i];
    pcnn_layer_info &f = infos[i];
    std::memset(&f, 0, sizeof f);
    f.kind = ly.d.kind;
    f.in_c = ly.in_c;
    f.in_h = ly.in_h;
    f.in_w = ly.in_w;
    f.out_c = ly.out_c;
    f.out_h = ly.out_h;
    f.out_w = ly.out_w;
    f.groups = ly.gemm ? ly.d.groups : 1;
    if (ly.d.kind == PCNN_CONV) {
      f.gemm_m = (long long)batch * ly.out_h * ly.out_w;
      f.gemm_n = ly.d.out_channels / ly.d.groups;
      f.gemm_k = ly.d.kernel * ly.d.kernel * (ly.in_c / ly.d.groups);
    } else if (ly.d.kind == PCNN_FC) {
      f.gemm_m = batch;
      f.gemm_n = ly.d.out_channels;
      f.gemm_k = ly.in_c * ly.in_h * ly.in_w;
    }
    f.flops = f.flops_exact = layer_flops_exact(ly, batch);
    f.bytes = layer_bytes(ly, batch, desc->precision, i == n_layers - 1);
    f.engine = ly.gemm ? (desc->precision == PCNN_FP32_SIMT ? 0 : 1) : 2;
  }
  return PCNN_OK;
}

pcnn_status pcnn_create_net(const pcnn_net_desc *desc, const pcnn_layer_desc *layers,
                            int n_layers, const float *const *weights,
                            const float *const *biases, pcnn_net **out) {
  if (!out) return fail(PCNN_ERR_INVALID_ARGUMENT, "out is null");
  *out = nullptr;
  if (!desc || desc->max_batch <= 0) return fail(PCNN_ERR_INVALID_ARGUMENT, "bad max_batch");
  std::unique_ptr<pcnn_net> net(new pcnn_net());
  net->desc = *desc;
  pcnn_status s = infer_shapes(desc, layers, n_layers, net->layers);
  if (s != PCNN_OK) return s;
  for (int i = 0; i < n_layers; ++i)
    if (net->layers[i].gemm && (!weights || !weights[i]))
      return fail(PCNN_ERR_INVALID_ARGUMENT, "missing weights for layer " + std::to_string(i));
  // device
  int ndev = 0;
  if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev <= desc->device || desc->device < 0) {
    cudaGetLastError();
    return fail(PCNN_ERR_CUDA, "no CUDA device " + std::to_string(desc->device));
  }
  CUDA_TRY(cudaSetDevice(desc->device));
  cudaDeviceProp prop;
  CUDA_TRY(cudaGetDeviceProperties(&prop, desc->device));
  if (prop.major != 10)
    return fail(PCNN_ERR_CUDA, std::string("device is not sm_100 (Blackwell): ") + prop.name);
  net->device = desc->device;
  net->num_sms = std::min(prop.multiProcessorCount, kMaxSMs);
  net->st = storage_of(desc->precision);
  net->in_cs = round_up(desc->in_channels, chunk_elems(desc->precision));
  net->occ_simt = simt_conv_occupancy();
  net->occ_lp = lrn_pool_occupancy(net->st);
  net->stage_h = desc->in_height;
  net->stage_w = desc->in_width;
  net->fuse_lrn_pool = !(desc->flags & PCNN_FLAG_NO_LRN_POOL_FUSION);
  net->conv_lrn_pm = (desc->flags & PCNN_FLAG_CONV_LRN_EPILOGUE) != 0;
  net->perf_im2col = (desc->flags & PCNN_FLAG_PERFORATION_IM2COL) != 0;
  net->per_row_windows = (desc->flags & PCNN_FLAG_PER_ROW_WINDOWS) != 0;
  if (desc->precision != PCNN_FP32_SIMT) {
    if (!get_encode_tiled() || !get_encode_im2col())
      return fail(PCNN_ERR_CUDA, "driver entry points cuTensorMapEncode{Tiled,Im2col} unavailable");
    CUDA_TRY(tc_init());
  }

  const int prec = desc->precision;
  const int esz = esz_of(net->st);
  const int B = desc->max_batch;
  // TMA slab alignment: a grouped conv whose channels per group are not a
  // multiple of 128 bytes reads its input with narrow (SW64/SW32) slabs.  When
  // its producer is an LRN / pooling layer, that producer writes each group
  // padded to a multiple of 128 bytes instead (zeros; packed weights are zero
  // there too), so the conv loads full SW128 slabs.
  const int slab128 = 128 / esz;
  // PCNN_FLAG_NARROW_SLABS: keep such groups unpadded and run the conv in
  // padded-layout mode on narrow (SW32 / SW64) slabs -- no K padding waste
  const bool narrow_pm = (desc->flags & PCNN_FLAG_NARROW_SLABS) != 0;
  if (prec != PCNN_FP32_SIMT && !narrow_pm) {
    for (int i = 1; i < n_layers; ++i) {
      Layer &ly = net->layers[i];
      Layer &pv = net->layers[i - 1];
      if (ly.d.kind != PCNN_CONV || ly.d.groups <= 1) continue;
      const int cg = ly.in_c / ly.d.groups;
      if ((cg % slab128) == 0 || ly.in_cs != ly.in_c) continue;
      if (pv.d.kind != PCNN_MAXPOOL && pv.d.kind != PCNN_AVGPOOL && pv.d.kind != PCNN_LRN) continue;
      pv.out_groups = ly.d.groups;
      pv.out_cg_pad = round_up(cg, slab128);
      pv.out_cs = ly.d.groups * pv.out_cg_pad;
      ly.in_cs = pv.out_cs;
    }
  }
  // Space-to-depth for a strided first conv (layout transform of a1): the
  // conv S x S / st on C channels becomes ceil(S/st) x ceil(S/st) / 1 on
  // st^2 C channels over an (Ho - 1 + S') x (Wo - 1 + S') grid whose origin
  // is shifted by -pad.  Same products, no K padding waste.
  std::vector<float> s2d_w;
  const Layer &l0 = net->layers[0];
  const bool no_s2d = (desc->flags & PCNN_FLAG_NO_SPACE_TO_DEPTH) != 0;
  const int k0 = l0.d.kernel;
  if (prec != PCNN_FP32_SIMT && l0.d.kind == PCNN_CONV && l0.d.groups == 1 &&
      desc->in_channels == 3 && (k0 == 3 || k0 == 5) && 3 * k0 * k0 <= 128 &&
      !no_s2d) {
    // im2col staging: W'[f][(r*S + s)*3 + c] = W[f][c][r][s], a 1x1 conv on Kp channels
    const int K = 3 * k0 * k0, F = l0.d.out_channels;
    const int Kp = K <= 64 / esz * 2 ? round_up(K, 64 / esz) : round_up(K, 128 / esz);
    net->stage_im2col = 1;
    net->stage_c = K;
    net->stage_h = l0.out_h;
    net->stage_w = l0.out_w;
    net->in_cs = Kp;
    s2d_w.assign((size_t)F * K, 0.f);
    for (int f = 0; f < F; ++f)
      for (int c = 0; c < 3; ++c)
        for (int r = 0; r < k0; ++r)
          for (int q = 0; q < k0; ++q)
            s2d_w[(size_t)f * K + (r * k0 + q) * 3 + c] = weights[0][(((size_t)f * 3 + c) * k0 + r) * k0 + q];
  } else if (l0.d.kind == PCNN_CONV && l0.d.groups == 1 && l0.d.stride >= 2 && l0.d.stride <= 8 &&
      !no_s2d) {
    const int st2 = l0.d.stride, S = l0.d.kernel, Sp = (S + st2 - 1) / st2;
    const int C = desc->in_channels, Cp = st2 * st2 * C, F = l0.d.out_channels;
    net->stage_blk = st2;
    net->stage_pad = l0.d.pad;
    net->stage_c = Cp;
    net->stage_h = l0.out_h - 1 + Sp;
    net->stage_w = l0.out_w - 1 + Sp;
    net->in_cs = round_up(Cp, prec == PCNN_FP32_SIMT ? chunk_elems(prec) : slab128);
    s2d_w.assign((size_t)F * Cp * Sp * Sp, 0.f);
    for (int f = 0; f < F; ++f)
      for (int c = 0; c < C; ++c)
        for (int r = 0; r < S; ++r)
          for (int q = 0; q < S; ++q) {
            const int cp = ((r % st2) * st2 + (q % st2)) * C + c;
            s2d_w[(((size_t)f * Cp + cp) * Sp + r / st2) * Sp + q / st2] =
                weights[0][(((size_t)f * C + c) * S + r) * S + q];
          }
  }
  // Padded-layout ("shifted window") convs, ConvGeom::pm: a stride-1 'same'
  // conv whose input and output share one zero-haloed grid loads, per filter
  // row, one TMA window of 128 + S - 1 rows that feeds all S taps -- S times
  // fewer A bytes than im2col boxes.  Chosen per net: the conv's producer and
  // consumer must read / write the halo layout (pools and pm convs of the same
  // halo do; a staged-im2col first layer joins as a 1 x 1 pm conv), channels
  // per group must fill 128 B slabs, and the halo may add at most 40% rows.
  const int n = n_layers;
  {
    const bool allow = prec != PCNN_FP32_SIMT && !(desc->flags & PCNN_FLAG_NO_PADDED_LAYOUT);
    // halo rows are computed and discarded: up to 40% extra MMA rows still
    // beats im2col boxes (S x fewer A bytes through the tiled-TMA path,
    // measured 2x faster per byte than im2col mode on B200)
    const char *eh = exp_env("PCNN_PM_MAX_HALO");
    const double pm_max_halo = eh ? atof(eh) : 1.40;
    auto kind = [&](int j) { return net->layers[j].d.kind; };
    auto is_pool = [&](int j) { return kind(j) == PCNN_MAXPOOL || kind(j) == PCNN_AVGPOOL; };
    std::vector<int> pmh(n, 0);
    if (allow) {
      for (int i = 1; i < n; ++i) {
        const Layer &ly = net->layers[i];
        if (ly.d.kind != PCNN_CONV) continue;
        const int S = ly.d.kernel, P = ly.d.pad, g = ly.d.groups;
        if (ly.d.stride != 1 || S != 2 * P + 1 || P < 1 || P > 3 || ly.in_cs % g) continue;
        const int sb = tc_slab_bytes(net->st, ly.in_cs / g);
        if (sb == 0 || (sb != 128 && !narrow_pm)) continue;
        // shared-halo grid: P zero rows / columns per image row / image
        if ((double)(ly.in_h + P) * (ly.in_w + P) > pm_max_halo * ly.in_h * ly.in_w) continue;
        pmh[i] = P;
      }
      for (bool changed = true; changed;) {
        changed = false;
        if (net->stage_blk > 1 && n > 1 && kind(0) == PCNN_CONV) {
          // space-to-depth first conv: Sp x Sp, stride 1, pad 0 on the staged
          // grid -- a 'valid' pm conv when Sp is odd and its consumer reads a halo
          const int Sp = (net->layers[0].d.kernel + net->stage_blk - 1) / net->stage_blk;
          const int hh = (Sp % 2 == 1 && Sp > 1 && Sp <= 7 &&
                          tc_slab_bytes(net->st, net->in_cs) == 128 &&
                          (is_pool(1) || kind(1) == PCNN_LRN))
                             ? (Sp - 1) / 2 : 0;
          if (pmh[0] != hh) {
            pmh[0] = hh;
            changed = true;
          }
        }
        if (net->stage_im2col && n > 1) {
          const int h = kind(1) == PCNN_CONV && tc_slab_bytes(net->st, net->in_cs) ? pmh[1] : 0;
          if (pmh[0] != h) {
            pmh[0] = h;
            changed = true;
          }
        }
        for (int i = 1; i < n; ++i) {
          if (!pmh[i]) continue;
          auto nb_ok = [&](int j) {
            return j >= 0 && j < n && (is_pool(j) || (kind(j) == PCNN_CONV && pmh[j] == pmh[i]));
          };
          // an LRN consumer reads the halo grid too (its kernel takes an input halo)
          auto cons_ok = [&](int j) { return nb_ok(j) || (j < n && kind(j) == PCNN_LRN); };
          if (!nb_ok(i - 1) || !cons_ok(i + 1)) {
            pmh[i] = 0;
            changed = true;
          }
        }
      }
    }
    for (int i = 0; i < n; ++i) {
      Layer &ly = net->layers[i];
      ly.in_halo = i > 0 ? net->layers[i - 1].out_halo : (net->stage_blk > 1 ? 0 : pmh[0]);
      ly.pm_halo = pmh[i];
      // shared-halo layouts: a 'same' pm conv keeps its grid (halo P); the
      // 'valid' space-to-depth first conv computes its output on the staged
      // grid, i.e. the output's halo is Sp - 1 = 2 pmh
      if (pmh[i]) ly.out_halo = (i == 0 && net->stage_blk > 1) ? 2 * pmh[i] : pmh[i];
      else if (is_pool(i) && i + 1 < n && kind(i + 1) == PCNN_CONV) ly.out_halo = pmh[i + 1];
      else if (kind(i) == PCNN_LRN && i > 0 && pmh[i - 1] && i + 1 < n && is_pool(i + 1))
        ly.out_halo = net->layers[i - 1].out_halo;   // keeps the conv's layout (conv + LRN may fuse)
      else ly.out_halo = 0;
    }
  }
  const int h0 = net->layers[0].in_halo;
  size_t act = (size_t)B * (net->stage_h + h0) * (net->stage_w + h0) * net->in_cs * esz;
  for (int i = 0; i < n; ++i) {
    Layer &ly = net->layers[i];
    act = std::max(act, (size_t)B * (ly.out_h + ly.out_halo) * (ly.out_w + ly.out_halo) *
                            ly.out_cs * esz);
    if (ly.gemm) {
      const bool final_fc = (i == n - 1) && ly.d.kind == PCNN_FC;
      const int mode = final_fc ? OUT_F32
                                : (net->st == ST_BF16 ? OUT_BF16
                                                      : (prec == PCNN_TF32 ? OUT_F32_TF32 : OUT_F32));
      const bool is_fc = ly.d.kind == PCNN_FC;
      if (i == 0 && net->stage_im2col) {
        s = build_stage(ly.exact, ly, prec, ly.d.out_channels, 1, 1, 1, 0, ly.d.relu,
                        net->stage_c, net->stage_h, net->stage_w, net->in_cs, false,
                        s2d_w.data(), biases ? biases[i] : nullptr, mode, ly.pm_halo);
      } else if (i == 0 && net->stage_blk > 1) {
        const int Sp = (ly.d.kernel + net->stage_blk - 1) / net->stage_blk;
        s = build_stage(ly.exact, ly, prec, ly.d.out_channels, 1, Sp, 1, 0, ly.d.relu,
                        net->stage_c, net->stage_h, net->stage_w, net->in_cs, false,
                        s2d_w.data(), biases ? biases[i] : nullptr, mode, ly.pm_halo,
                        ly.pm_halo > 0);
      } else {
        s = build_stage(ly.exact, ly, prec, ly.d.out_channels, is_fc ? 1 : ly.d.groups,
                        is_fc ? 1 : ly.d.kernel, is_fc ? 1 : ly.d.stride,
                        is_fc ? 0 : ly.d.pad, ly.d.relu, ly.in_c, ly.in_h, ly.in_w,
                        ly.in_cs, is_fc, weights[i], biases ? biases[i] : nullptr, mode,
                        ly.pm_halo);
      }
      if (s != PCNN_OK) {
        for (auto &l2 : net->layers) l2.exact.release();
        return fail(s, "layer " + std::to_string(i) + ": " + g_err);
      }
      if (ly.d.kind == PCNN_CONV) {
        const size_t cnt = (size_t)ly.d.out_channels * (ly.in_c / ly.d.groups) * ly.d.kernel *
                           ly.d.kernel;
        ly.host_w.assign(weights[i], weights[i] + cnt);
      }
    }
    CUDA_TRY(cudaMalloc(&ly.d_ctr, sizeof(unsigned long long) * 3 * (1 + kMaxSMs)));
    CUDA_TRY(cudaMemset(ly.d_ctr, 0, sizeof(unsigned long long) * 3 * (1 + kMaxSMs)));
    CUDA_TRY(cudaMalloc(&ly.d_census, 32));
    CUDA_TRY(cudaMemset(ly.d_census, 0, 32));
  }
  net->act_bytes = act;
  for (int k = 0; k < 3; ++k) {
    if (cudaMalloc(&net->d_act[k], act) != cudaSuccess) {
      cudaGetLastError();
      return fail(PCNN_ERR_OUT_OF_MEMORY, "activation arena");
    }
  }
  const Layer &last = net->layers.back();
  net->out_elems = last.out_c * last.out_h * last.out_w;
  *out = net.release();
  return PCNN_OK;
}

static void destroy_graphs(pcnn_net *net) {
  for (auto &kv : net->graphs) cudaGraphExecDestroy(kv.second);
  net->graphs.clear();
}

pcnn_status pcnn_destroy_net(pcnn_net *net) {
  if (!net) return PCNN_OK;
  cudaSetDevice(net->device);
  destroy_graphs(net);
  for (auto *lst : {&net->timing_sets, &net->timing_free})
    for (auto &ev : *lst)
      for (auto e : ev) cudaEventDestroy(e);
  for (auto &ly : net->layers) {
    ly.exact.release();
    ly.r1.release();
    ly.r2.release();
    ly.pf.release();
    if (ly.d_ctr) cudaFree(ly.d_ctr);
    if (ly.d_census) cudaFree(ly.d_census);
  }
  for (auto &p : net->d_act)
    if (p) cudaFree(p);
  if (net->d_ws) cudaFree(net->d_ws);
  if (net->copy_stream) cudaStreamDestroy(net->copy_stream);
  for (auto &e : net->ev_copy)
    if (e) cudaEventDestroy(e);
  if (net->d_host_in) cudaFree(net->d_host_in);
  if (net->d_host_u8) cudaFree(net->d_host_u8);
  if (net->d_mean) cudaFree(net->d_mean);
  if (net->d_host_out) cudaFree(net->d_host_out);
  if (net->d_host_p) cudaFree(net->d_host_p);
  if (net->d_host_h) cudaFree(net->d_host_h);
  delete net;
  return PCNN_OK;
}

pcnn_status pcnn_num_layers(const pcnn_net *net, int *n) {
  if (!net || !n) return fail(PCNN_ERR_INVALID_ARGUMENT, "null");
  *n = (int)net->layers.size();
  return PCNN_OK;
}

pcnn_status pcnn_output_size(const pcnn_net *net, int *n) {
  if (!net || !n) return fail(PCNN_ERR_INVALID_ARGUMENT, "null");
  *n = net->out_elems;
  return PCNN_OK;
}

pcnn_status pcnn_set_variant(pcnn_net *net, int layer, int variant, int rank) {
  if (!net || layer < 0 || layer >= (int)net->layers.size())
    return fail(PCNN_ERR_INVALID_ARGUMENT, "bad net / layer");
  Layer &ly = net->layers[layer];
  if (variant == PCNN_VARIANT_EXACT) {
    if (ly.variant != PCNN_VARIANT_EXACT || ly.perf_sh * ly.perf_sw > 1) net->version++;
    ly.variant = PCNN_VARIANT_EXACT;
    ly.rank = 0;
    ly.perf_sh = ly.perf_sw = 1;
    return PCNN_OK;
  }
  if (ly.perf_sh * ly.perf_sw > 1)
    return fail(PCNN_ERR_UNSUPPORTED, "rank variant of a perforated layer (set EXACT first)");
  if (variant != PCNN_VARIANT_RANK) return fail(PCNN_ERR_INVALID_ARGUMENT, "bad variant");
  if (ly.d.kind != PCNN_CONV)
    return fail(PCNN_ERR_UNSUPPORTED, "rank variant is implemented for conv layers");
  if (layer == 0 && (net->stage_im2col || net->stage_blk > 1))
    return fail(PCNN_ERR_UNSUPPORTED,
                "rank variant of a first conv whose input is staged (im2col / space-to-depth)");
  const int g = ly.d.groups, Nfg = ly.d.out_channels / g, Cg = ly.in_c / g,
            S = ly.d.kernel, K = Cg * S * S;
  const int rmax = std::min(Nfg, K);
  if (rank < 1 || rank > rmax)
    return fail(PCNN_ERR_INVALID_ARGUMENT, "rank out of [1, min(N_f/g, K)]");
  CUDA_TRY(cudaSetDevice(net->device));
  if (ly.svd.empty()) {
    for (int gi = 0; gi < g; ++gi) {
      std::vector<double> Wg((size_t)Nfg * K);
      for (size_t i = 0; i < Wg.size(); ++i) Wg[i] = ly.host_w[(size_t)gi * Nfg * K + i];
      ly.svd.push_back(svd_rows(Wg, Nfg, K));
    }
  }
  // A = U_r Sigma_r  [g][Nfg][r],  B = V_r^T  [g][r][K]  (K in OIHW (c, r, s) order)
  std::vector<float> A((size_t)g * Nfg * rank), Bm((size_t)g * rank * K);
  for (int gi = 0; gi < g; ++gi) {
    const Svd &sv = ly.svd[gi];
    for (int f = 0; f < Nfg; ++f)
      for (int a = 0; a < rank; ++a)
        A[((size_t)gi * Nfg + f) * rank + a] = (float)(sv.U[(size_t)f * Nfg + a] * sv.sigma[a]);
    for (int a = 0; a < rank; ++a)
      for (int k = 0; k < K; ++k)
        Bm[((size_t)gi * rank + a) * K + k] = (float)sv.Vt[(size_t)a * K + k];
  }
  return build_rank_stages(net, ly, rank, A.data(), Bm.data());
}

pcnn_status pcnn_set_perforation(pcnn_net *net, int layer, int sh, int sw) {
  if (!net || layer < 0 || layer >= (int)net->layers.size() || sh < 1 || sw < 1 || sh > 4 ||
      sw > 4)
    return fail(PCNN_ERR_INVALID_ARGUMENT, "bad net / layer / perforation steps (1..4)");
  Layer &ly = net->layers[layer];
  if (ly.d.kind != PCNN_CONV)
    return fail(PCNN_ERR_UNSUPPORTED, "perforation is defined for conv layers (P:328)");
  if (sh * sw == 1) {
    if (ly.perf_sh * ly.perf_sw > 1) net->version++;
    ly.perf_sh = ly.perf_sw = 1;
    ly.pf.release();
    return PCNN_OK;
  }
  if (ly.variant != PCNN_VARIANT_EXACT)
    return fail(PCNN_ERR_UNSUPPORTED, "perforation of a rank-r layer (set EXACT first)");
  if (net->desc.precision == PCNN_FP32_SIMT)
    return fail(PCNN_ERR_UNSUPPORTED, "perforation runs on the tcgen05 engine (BF16 / TF32)");
  if (layer == 0 && (net->stage_im2col || net->stage_blk > 1))
    return fail(PCNN_ERR_UNSUPPORTED,
                "perforation of a first conv whose input is staged (im2col / space-to-depth)");
  if (ly.in_halo > 0 && ly.in_halo < ly.d.pad)
    return fail(PCNN_ERR_UNSUPPORTED, "input halo narrower than the conv padding");
  CUDA_TRY(cudaSetDevice(net->device));
  const int mode = ly.exact.g.out_mode;
  // rows only, on a padded-layout layer whose grid rows fit one MMA tile:
  // the kept rows run in padded-layout mode (pm = 2, row-strided windows)
  const bool pm2 = sw == 1 && ly.exact.g.pm == 1 && ly.pm_halo > 0 &&
                   ly.exact.g.wv + 2 * ly.exact.g.pad <= 128 && !net->perf_im2col;
  pcnn_status s = build_stage(ly.pf, ly, net->desc.precision, ly.d.out_channels, ly.d.groups,
                              ly.d.kernel, ly.d.stride, ly.d.pad, ly.d.relu, ly.in_c, ly.in_h,
                              ly.in_w, ly.in_cs, false, ly.host_w.data(), nullptr, mode,
                              pm2 ? ly.pm_halo : 0);
  if (s != PCNN_OK) return s;
  CUDA_TRY(cudaMemcpy(ly.pf.d_bias, ly.exact.d_bias,
                      sizeof(float) * ((size_t)round_up(ly.d.out_channels, 256) + 256),
                      cudaMemcpyDeviceToDevice));
  ConvGeom &g = ly.pf.g;
  g.psh = sh;
  g.psw = sw;
  g.out_cs = ly.out_cs;
  if (pm2) {
    g.pm = 2;
    g.hk = (ly.out_h + sh - 1) / sh;
    g.nseg = 128 / (g.wv + 2 * g.pad);   // segments: grid columns -pad .. wv + pad
    g.tpi = (g.hk + g.nseg - 1) / g.nseg;
  } else {
    g.ih = ly.in_halo;
    g.Ho = (ly.out_h + sh - 1) / sh;      // kept rows / columns
    g.Wo = (ly.out_w + sw - 1) / sw;
  }
  ly.perf_sh = sh;
  ly.perf_sw = sw;
  net->version++;
  return PCNN_OK;
}

// FC rank-r (the conv form with S = 1): stage 1 = FC K -> r
// with B's rows (CHW-ordered columns, permuted like the exact fc), stage 2 =
// FC r -> N with A + bias (+ ReLU).
static pcnn_status build_rank_stages_fc(pcnn_net *net, Layer &ly, int r, const float *A,
                                        const float *Bf) {
  const auto &d = ly.d;
  const int prec = net->desc.precision, st = net->st, N = d.out_channels;
  const size_t K = (size_t)ly.in_c * ly.in_h * ly.in_w;
  const int rs = round_up(r, 64);                 // one full K-block of stage 2
  std::vector<float> w1((size_t)rs * K, 0.f), w2((size_t)N * rs, 0.f);
  std::memcpy(w1.data(), Bf, sizeof(float) * (size_t)r * K);
  for (int f = 0; f < N; ++f)
    for (int a = 0; a < r; ++a) w2[(size_t)f * rs + a] = A[(size_t)f * r + a];
  const int mode1 = st == ST_BF16 ? OUT_BF16 : (prec == PCNN_TF32 ? OUT_F32_TF32 : OUT_F32);
  pcnn_status s1 = build_stage(ly.r1, ly, prec, rs, 1, 1, 1, 0, 0, ly.in_c, ly.in_h, ly.in_w,
                               ly.in_cs, true, w1.data(), nullptr, mode1);
  if (s1 != PCNN_OK) return s1;
  const GemmStage &ex = ly.exact;
  pcnn_status s2 = build_stage(ly.r2, ly, prec, N, 1, 1, 1, 0, d.relu, rs, 1, 1, rs, true,
                               w2.data(), nullptr, ex.g.out_mode);
  if (s2 != PCNN_OK) return s2;
  CUDA_TRY(cudaMemcpy(ly.r2.d_bias, ex.d_bias, sizeof(float) * N, cudaMemcpyDeviceToDevice));
  ly.rank = r;
  ly.variant = PCNN_VARIANT_RANK;
  net->version++;
  return PCNN_OK;
}

pcnn_status pcnn_set_variant_factors(pcnn_net *net, int layer, int rank, const float *A,
                                     const float *B) {
  if (!net || layer < 0 || layer >= (int)net->layers.size() || !A || !B)
    return fail(PCNN_ERR_INVALID_ARGUMENT, "bad arguments");
  Layer &ly = net->layers[layer];
  if (ly.d.kind != PCNN_CONV && ly.d.kind != PCNN_FC)
    return fail(PCNN_ERR_UNSUPPORTED, "conv / fc layers only");
  if (rank < 1 || rank > 4096) return fail(PCNN_ERR_INVALID_ARGUMENT, "bad rank");
  if (ly.perf_sh * ly.perf_sw > 1)
    return fail(PCNN_ERR_UNSUPPORTED, "rank variant of a perforated layer (set EXACT first)");
  CUDA_TRY(cudaSetDevice(net->device));
  if (ly.d.kind == PCNN_FC) {
    if (rank > std::min<long long>(ly.d.out_channels, (long long)ly.in_c * ly.in_h * ly.in_w))
      return fail(PCNN_ERR_INVALID_ARGUMENT, "rank out of [1, min(N, K)]");
    return build_rank_stages_fc(net, ly, rank, A, B);
  }
  // the same guards as pcnn_set_variant: a staged first conv reads the
  // space-to-depth / im2col grid, not the logical input the factors refer to
  if (layer == 0 && (net->stage_im2col || net->stage_blk > 1))
    return fail(PCNN_ERR_UNSUPPORTED,
                "rank variant of a first conv whose input is staged (im2col / space-to-depth)");
  {
    const int g = ly.d.groups, Nfg = ly.d.out_channels / g;
    const int K = (ly.in_c / g) * ly.d.kernel * ly.d.kernel;
    if (rank > std::min(Nfg, K)) return fail(PCNN_ERR_INVALID_ARGUMENT, "rank out of [1, min(N_f/g, K)]");
    // stage 1 writes g * round_up(r, chunk) channels on the layer's output grid
    // into the arena's third buffer
    const size_t s1 = (size_t)net->desc.max_batch * (ly.out_h + ly.out_halo) *
                      (ly.out_w + ly.out_halo) * g *
                      round_up(rank, chunk_elems(net->desc.precision)) * esz_of(net->st);
    if (s1 > net->act_bytes)
      return fail(PCNN_ERR_UNSUPPORTED, "rank-r intermediate larger than the activation arena");
  }
  return build_rank_stages(net, ly, rank, A, B);
}

pcnn_status pcnn_set_sm_budget(pcnn_net *net, int layer, int n_sms, int ctas_per_sm) {
  if (!net || layer < 0 || layer >= (int)net->layers.size() || n_sms < 0 || ctas_per_sm < 0)
    return fail(PCNN_ERR_INVALID_ARGUMENT, "bad arguments");
  Layer &ly = net->layers[layer];
  ly.n_sms = n_sms >= net->num_sms ? 0 : n_sms;
  ly.tlp = ctas_per_sm;
  net->version++;
  return PCNN_OK;
}

pcnn_status pcnn_set_layer_plan(pcnn_net *net, int layer, int cta_group, int m_sub) {
  if (!net || layer < 0 || layer >= (int)net->layers.size())
    return fail(PCNN_ERR_INVALID_ARGUMENT, "bad net / layer");
  if (cta_group < 0 || cta_group > 2 || m_sub < 0 || m_sub > 2)
    return fail(PCNN_ERR_INVALID_ARGUMENT, "cta_group and m_sub must be 0, 1 or 2");
  Layer &ly = net->layers[layer];
  if (!ly.gemm || net->desc.precision == PCNN_FP32_SIMT)
    return fail(PCNN_ERR_UNSUPPORTED, "tile override applies to tcgen05 GEMM layers");
  ly.plan_cg = cta_group;
  ly.plan_msub = m_sub;
  net->version++;
  return PCNN_OK;
}

// eq. 12 on B200 (reading R12 / NEXT-3): t(n) = t_launch + nInvocations(n) x
// t_unit.  The paper's form FLOPs / (peakFlops x optSM x rEC x FMA share) is
// the per-wave term summed over full waves; on B200 a layer's latency also
// carries a fixed cost per launch (launch, CTA rasterisation, barrier / TMEM
// setup, pipeline fill, epilogue drain) that dominates at small batch.  The
// per-unit time comes from the planner's own cost model (operand bytes at the
// measured L2->SM rate vs. MMA cycles per K-block); the two constants per
// kernel class were fitted to measured per-layer latencies over n in
// {8..148} and B in {1, 64, 256} (tools/time_model_fit.py,
// profiles/r02_time_model_fit.json).
struct TimeModel { double launch_us, unit_scale; };
static TimeModel time_model_class(const pcnn_layer_info &f) {
  if (f.kind != PCNN_CONV && f.kind != PCNN_FC) return {kT0Simt, 1.0};
  if (f.engine == 0) return {kT0Simt, 1.0};
  if (f.a_mode == 3) return {kT0Fc, kScaleFc};
  return {kT0Conv, kScaleConv};
}

static pcnn_status layer_time_model(pcnn_net *net, int layer, int batch, int n_sms,
                                    pcnn_budget_plan *bp) {
  std::memset(bp, 0, sizeof *bp);
  Layer &ly = net->layers[layer];
  const int nsms = net->num_sms;
  const int n = n_sms <= 0 ? nsms : std::min(n_sms, nsms);
  bp->opt_sm = nsms;
  bp->cta_group = 1;
  bp->opt_tlp = 1;
  // the plan on the whole device (the budget in effect must not change it)
  const int save_sms = ly.n_sms, save_tlp = ly.tlp;
  ly.n_sms = 0;
  ly.tlp = 0;
  pcnn_layer_info f;
  pcnn_status s = pcnn_query_layer(net, layer, batch, &f);
  ly.n_sms = save_sms;
  ly.tlp = save_tlp;
  if (s != PCNN_OK) return s;
  const TimeModel tm = time_model_class(f);
  bp->t_launch_us = tm.launch_us;
  if (!ly.gemm) {
    // HBM-bound: the bytes at min(HBM, n x the per-SM streaming rate)
    const double bw = std::min(6.5e12, n * 60e9);
    bp->t_unit_us = f.bytes / bw * 1e6;
    bp->t_model_us = tm.launch_us + bp->t_unit_us;
    return PCNN_OK;
  }
  const int cg = std::max(1, f.cta_group);
  const long long G = f.tiles * std::max(1, f.splits);
  const int tlp = f.engine == 1 ? 1 : std::max(1, net->occ_simt);
  const long long slots = nsms / cg;                       // SMs in tile units
  const long long inv = (G + (long long)tlp * slots - 1) / ((long long)tlp * slots);   // eq. 8
  long long p = 1;                                        // eq. 11: the fewest units
  while (p < slots && (G + (long long)tlp * p - 1) / ((long long)tlp * p) != inv) ++p;
  bp->grid_size = G;
  bp->opt_tlp = tlp;
  bp->cta_group = cg;
  bp->opt_sm = (int)(p * cg);
  // eq. 8 at the budget n (FC units need their whole K-split group at once)
  long long slots_n = std::max<long long>(1, n / cg);
  if (f.a_mode == 3) slots_n = std::max<long long>(f.splits, slots_n / f.splits * f.splits);
  const long long inv_n = (G + (long long)tlp * slots_n - 1) / ((long long)tlp * slots_n);
  bp->n_invocations = (int)(n_sms <= 0 ? inv : inv_n);
  bp->t_unit_us = f.t_unit_us * tm.unit_scale;
  bp->t_model_us = tm.launch_us + bp->n_invocations * bp->t_unit_us;
  return PCNN_OK;
}

pcnn_status pcnn_plan_budget(const pcnn_net *cnet, int layer, int batch, pcnn_budget_plan *bp) {
  pcnn_net *net = const_cast<pcnn_net *>(cnet);
  if (!net || !bp || layer < 0 || layer >= (int)net->layers.size() || batch <= 0)
    return fail(PCNN_ERR_INVALID_ARGUMENT, "bad arguments");
  pcnn_status s = layer_time_model(net, layer, batch, 0, bp);
  if (s != PCNN_OK) return s;
  // t_model_us at opt_sm: eq. 11 keeps nInvocations, so the time is the
  // whole-device time by construction
  return PCNN_OK;
}

pcnn_status pcnn_model_layer_time(const pcnn_net *cnet, int layer, int batch, int n_sms,
                                  double *t_us) {
  pcnn_net *net = const_cast<pcnn_net *>(cnet);
  if (!net || !t_us || layer < 0 || layer >= (int)net->layers.size() || batch <= 0 || n_sms < 0)
    return fail(PCNN_ERR_INVALID_ARGUMENT, "bad arguments");
  pcnn_budget_plan bp;
  pcnn_status s = layer_time_model(net, layer, batch, n_sms, &bp);
  if (s != PCNN_OK) return s;
  *t_us = bp.t_model_us;
  return PCNN_OK;
}

pcnn_status pcnn_query_layer(const pcnn_net *cnet, int layer, int batch, pcnn_layer_info *f) {
  pcnn_net *net = const_cast<pcnn_net *>(cnet);
  if (!net || !f || layer < 0 || layer >= (int)net->layers.size() || batch <= 0)
    return fail(PCNN_ERR_INVALID_ARGUMENT, "bad arguments");
  Layer &ly = net->layers[layer];
  std::memset(f, 0, sizeof *f);
  f->splits = 1;
  f->kind = ly.d.kind;
  f->in_c = ly.in_c;
  f->in_h = ly.in_h;
  f->in_w = ly.in_w;
  f->out_c = ly.out_c;
  f->out_h = ly.out_h;
  f->out_w = ly.out_w;
  f->groups = ly.gemm ? ly.d.groups : 1;
  f->flops_exact = layer_flops_exact(ly, batch);
  f->flops = layer_flops_variant(ly, batch);
  f->bytes = layer_bytes(ly, batch, net->desc.precision, layer == (int)net->layers.size() - 1);
  f->variant = ly.variant;
  f->rank = ly.rank;
  f->n_sms = effective_sms(net, ly);
  f->tlp = ly.tlp;
  f->engine = 2;
  f->halo_in = ly.in_halo;
  f->halo_out = ly.out_halo;
  if (ly.gemm) {
    GemmStage &gs = ly.variant == PCNN_VARIANT_RANK ? ly.r1 : ly.exact;
    f->gemm_m = (long long)batch * gs.g.Ho * gs.g.Wo;
    f->gemm_n = ly.exact.g.Nfg;
    f->gemm_k = ly.d.kind == PCNN_CONV ? ly.d.kernel * ly.d.kernel * (ly.in_c / ly.d.groups)
                                       : ly.in_c * ly.in_h * ly.in_w;
    float lp[4];
    const bool fl = fuse_conv_lrn(net, layer);
    if (fl) lrn_params(net->layers[layer + 1], lp);
    GemmStage &ps = ly.perf_sh * ly.perf_sw > 1 ? ly.pf
                    : (ly.variant == PCNN_VARIANT_RANK ? ly.r2 : ly.exact);
    pcnn_status s = run_stage(net, ly, ps, batch, nullptr, nullptr, 0, nullptr, f, nullptr,
                              fl ? lp : nullptr);
    if (s != PCNN_OK) return s;
    const long long maxb = (long long)f->n_sms * std::max(f->tlp, 1);
    const long long waves = (f->tiles + maxb - 1) / maxb;
    f->util = (double)f->tiles / ((double)waves * maxb);                 // eq. 6
    const long long M = f->gemm_m, N = f->gemm_n;
    const long long mt = (M + f->tile_m - 1) / f->tile_m, nt = (N + f->tile_n - 1) / f->tile_n;
    f->rec = (double)M * N / ((double)mt * nt * f->tile_m * f->tile_n);   // eq. 9
  }
  return PCNN_OK;
}

pcnn_status pcnn_infer(pcnn_net *net, const float *d_images, int batch, float *d_out,
                       float *d_probs, float *d_entropy, void *stream) {
  if (!net || !d_images || !d_out) return fail(PCNN_ERR_INVALID_ARGUMENT, "null pointer");
  if (batch <= 0) return fail(PCNN_ERR_INVALID_ARGUMENT, "batch must be positive");
  if (batch > net->desc.max_batch) return fail(PCNN_ERR_BATCH_TOO_LARGE, "batch > max_batch");
  CUDA_TRY(cudaSetDevice(net->device));
  {
    pcnn_status r = ensure_workspace(net, batch);
    if (r != PCNN_OK) return r;
  }
  cudaStream_t s = (cudaStream_t)stream;
  if (net->timing) {
    std::vector<cudaEvent_t> ev;
    if (!net->timing_free.empty()) {
      ev = std::move(net->timing_free.back());
      net->timing_free.pop_back();
    } else {
      ev.resize(net->layers.size() + 1);
      for (auto &e : ev) CUDA_TRY(cudaEventCreate(&e));
    }
    pcnn_status r = enqueue_all(net, d_images, batch, d_out, d_probs, d_entropy, s, &ev);
    net->timing_sets.push_back(std::move(ev));
    return r;
  }
  if (!net->use_graphs || net->census || s == nullptr)
    return enqueue_all(net, d_images, batch, d_out, d_probs, d_entropy, s, nullptr);
  pcnn_net::GraphKey key{batch, d_images, d_out, d_probs, d_entropy, s, net->version};
  auto it = net->graphs.find(key);
  if (it == net->graphs.end()) {
    if (net->graphs.size() > 64) destroy_graphs(net);
    CUDA_TRY(cudaStreamBeginCapture(s, cudaStreamCaptureModeThreadLocal));
    pcnn_status r = enqueue_all(net, d_images, batch, d_out, d_probs, d_entropy, s, nullptr);
    cudaGraph_t graph = nullptr;
    cudaError_t ce = cudaStreamEndCapture(s, &graph);
    if (r != PCNN_OK) {
      if (graph) cudaGraphDestroy(graph);
      return r;
    }
    if (ce != cudaSuccess) return fail(PCNN_ERR_CUDA, std::string("graph capture: ") + cudaGetErrorString(ce));
    cudaGraphExec_t exec = nullptr;
    ce = cudaGraphInstantiate(&exec, graph, 0);
    cudaGraphDestroy(graph);
    if (ce != cudaSuccess) return fail(PCNN_ERR_CUDA, std::string("graph instantiate: ") + cudaGetErrorString(ce));
    it = net->graphs.emplace(key, exec).first;
  }
  CUDA_TRY(cudaGraphLaunch(it->second, s));
  return PCNN_OK;
}

// pcnn_infer_host / pcnn_infer_host_u8: host images (fp32, or uint8 pixels
// converted on the device) -> library device buffers -> pcnn_infer, chunked
// so that the host->device copies overlap inference when they dominate.
static pcnn_status infer_host_impl(pcnn_net *net, const float *h_images,
                                   const unsigned char *h_pixels, const float *mean, float scale,
                                   int batch, float *h_out, float *h_probs, float *h_entropy,
                                   void *stream) {
  if (!net || !(h_images || h_pixels) || !h_out)
    return fail(PCNN_ERR_INVALID_ARGUMENT, "null pointer");
  if (batch <= 0 || batch > net->desc.max_batch)
    return fail(PCNN_ERR_BATCH_TOO_LARGE, "bad batch");
  CUDA_TRY(cudaSetDevice(net->device));
  const int C = net->desc.in_channels;
  const size_t in_elems = (size_t)C * net->desc.in_height * net->desc.in_width;
  const size_t maxb = net->desc.max_batch;
  if (!net->d_host_in) {
    CUDA_TRY(cudaMalloc(&net->d_host_in, sizeof(float) * in_elems * maxb));
    CUDA_TRY(cudaMalloc(&net->d_host_out, sizeof(float) * net->out_elems * maxb));
    CUDA_TRY(cudaMalloc(&net->d_host_p, sizeof(float) * net->out_elems * maxb));
    CUDA_TRY(cudaMalloc(&net->d_host_h, sizeof(float) * maxb));
  }
  cudaStream_t s = (cudaStream_t)stream;
  const bool u8 = h_pixels != nullptr;
  if (u8) {
    if (!net->d_host_u8) {
      CUDA_TRY(cudaMalloc(&net->d_host_u8, in_elems * maxb));
      CUDA_TRY(cudaMalloc(&net->d_mean, sizeof(float) * C));
    }
    std::vector<float> m(C, 0.f);
    if (mean) m.assign(mean, mean + C);
    CUDA_TRY(cudaMemcpyAsync(net->d_mean, m.data(), sizeof(float) * C, cudaMemcpyHostToDevice, s));
  }
  const size_t in_bytes = u8 ? 1 : sizeof(float);
  // When the images take long to cross PCIe (25-50 GB/s pinned) compared with the
  // inference (FLOPs at ~700 TFLOP/s), split the batch into 4 chunks: chunk
  // i+1's host->device copy (own stream) overlaps chunk i's inference.
  // Images are independent, so the chunks compute the same per-image results.
  double flops = 0;
  for (auto &ly : net->layers) flops += layer_flops_exact(ly, 1);
  const double h2d_img = in_bytes * in_elems / 50e9, comp_img = flops / 7e14;
  int k = (batch >= 64 && h2d_img > (u8 ? 0.25 : 2.0) * comp_img) ? 4 : 1;
  if (const char *e = exp_env("PCNN_H2D_CHUNKS")) k = std::max(1, std::min(4, atoi(e)));   // experiments
  const int chunk = (batch + k - 1) / k;
  if (k > 1 && !net->copy_stream) {
    CUDA_TRY(cudaStreamCreateWithFlags(&net->copy_stream, cudaStreamNonBlocking));
    for (auto &e : net->ev_copy) CUDA_TRY(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
  }
  if (k > 1) {     // copies start after the caller's prior work on `stream`
    CUDA_TRY(cudaEventRecord(net->ev_copy[4], s));
    CUDA_TRY(cudaStreamWaitEvent(net->copy_stream, net->ev_copy[4], 0));
  }
  for (int c = 0, b0 = 0; b0 < batch; ++c, b0 += chunk) {
    const int nb = std::min(chunk, batch - b0);
    if (u8)
      CUDA_TRY(cudaMemcpyAsync(net->d_host_u8 + (size_t)b0 * in_elems, h_pixels + (size_t)b0 * in_elems,
                               in_elems * nb, cudaMemcpyHostToDevice, k > 1 ? net->copy_stream : s));
    else
      CUDA_TRY(cudaMemcpyAsync(net->d_host_in + (size_t)b0 * in_elems, h_images + (size_t)b0 * in_elems,
                               sizeof(float) * in_elems * nb, cudaMemcpyHostToDevice,
                               k > 1 ? net->copy_stream : s));
    if (k > 1) CUDA_TRY(cudaEventRecord(net->ev_copy[c], net->copy_stream));
  }
  for (int c = 0, b0 = 0; b0 < batch; ++c, b0 += chunk) {
    const int nb = std::min(chunk, batch - b0);
    if (k > 1) CUDA_TRY(cudaStreamWaitEvent(s, net->ev_copy[c], 0));
    if (u8)
      CUDA_TRY(counted(launch_pixels_u8(net->d_host_u8 + (size_t)b0 * in_elems, net->d_mean, scale,
                                        net->d_host_in + (size_t)b0 * in_elems, nb, C,
                                        (int)(in_elems / C), s)));
    const size_t oo = (size_t)b0 * net->out_elems;
    pcnn_status r = pcnn_infer(net, net->d_host_in + (size_t)b0 * in_elems, nb,
                               net->d_host_out + oo, h_probs ? net->d_host_p + oo : nullptr,
                               h_entropy ? net->d_host_h + b0 : nullptr, stream);
    if (r != PCNN_OK) return r;
    CUDA_TRY(cudaMemcpyAsync(h_out + oo, net->d_host_out + oo, sizeof(float) * net->out_elems * nb,
                             cudaMemcpyDeviceToHost, s));
    if (h_probs)
      CUDA_TRY(cudaMemcpyAsync(h_probs + oo, net->d_host_p + oo,
                               sizeof(float) * net->out_elems * nb, cudaMemcpyDeviceToHost, s));
    if (h_entropy)
      CUDA_TRY(cudaMemcpyAsync(h_entropy + b0, net->d_host_h + b0, sizeof(float) * nb,
                               cudaMemcpyDeviceToHost, s));
  }
  CUDA_TRY(cudaStreamSynchronize(s));
  return PCNN_OK;
}

pcnn_status pcnn_infer_host(pcnn_net *net, const float *h_images, int batch, float *h_out,
                            float *h_probs, float *h_entropy, void *stream) {
  return infer_host_impl(net, h_images, nullptr, nullptr, 1.f, batch, h_out, h_probs, h_entropy,
                         stream);
}

pcnn_status pcnn_infer_host_u8(pcnn_net *net, const unsigned char *h_pixels, const float *mean,
                               float scale, int batch, float *h_out, float *h_probs,
                               float *h_entropy, void *stream) {
  if (!h_pixels) return fail(PCNN_ERR_INVALID_ARGUMENT, "null pointer");
  return infer_host_impl(net, nullptr, h_pixels, mean, scale, batch, h_out, h_probs, h_entropy,
                         stream);
}

pcnn_status pcnn_profile_layers(pcnn_net *net, const float *d_images, int batch, float *d_out,
                                int reps, float *layer_ms, float *total_ms, void *stream) {
  if (!net || !d_images || !d_out || !layer_ms || reps <= 0)
    return fail(PCNN_ERR_INVALID_ARGUMENT, "bad arguments");
  if (batch <= 0 || batch > net->desc.max_batch) return fail(PCNN_ERR_BATCH_TOO_LARGE, "bad batch");
  CUDA_TRY(cudaSetDevice(net->device));
  {
    pcnn_status r = ensure_workspace(net, batch);
    if (r != PCNN_OK) return r;
  }
  cudaStream_t s = (cudaStream_t)stream;
  const int n = (int)net->layers.size();
  std::vector<cudaEvent_t> ev(n + 1);
  cudaEvent_t e_begin, e_end;
  for (auto &e : ev) CUDA_TRY(cudaEventCreate(&e));
  CUDA_TRY(cudaEventCreate(&e_begin));
  CUDA_TRY(cudaEventCreate(&e_end));
  std::vector<double> acc(n, 0.0);
  double tot = 0;
  for (int r = 0; r < reps; ++r) {
    CUDA_TRY(cudaEventRecord(e_begin, s));
    pcnn_status st = enqueue_all(net, d_images, batch, d_out, nullptr, nullptr, s, &ev);
    if (st != PCNN_OK) return st;
    CUDA_TRY(cudaEventRecord(e_end, s));
    CUDA_TRY(cudaEventSynchronize(e_end));
    for (int i = 0; i < n; ++i) {
      float ms = 0;
      CUDA_TRY(cudaEventElapsedTime(&ms, ev[i], ev[i + 1]));
      acc[i] += ms;
    }
    float t = 0;
    CUDA_TRY(cudaEventElapsedTime(&t, e_begin, e_end));
    tot += t;
  }
  for (int i = 0; i < n; ++i) layer_ms[i] = (float)(acc[i] / reps);
  if (total_ms) *total_ms = (float)(tot / reps);
  for (auto &e : ev) cudaEventDestroy(e);
  cudaEventDestroy(e_begin);
  cudaEventDestroy(e_end);
  return PCNN_OK;
}

pcnn_status pcnn_set_layer_timing(pcnn_net *net, int enable) {
  if (!net) return fail(PCNN_ERR_INVALID_ARGUMENT, "null net");
  net->timing = enable != 0;
  return PCNN_OK;
}

pcnn_status pcnn_read_layer_timing(pcnn_net *net, float *layer_ms, int *n_steps) {
  if (!net || !layer_ms) return fail(PCNN_ERR_INVALID_ARGUMENT, "null argument");
  CUDA_TRY(cudaSetDevice(net->device));
  const int n = (int)net->layers.size();
  std::vector<double> acc(n, 0.0);
  for (auto &ev : net->timing_sets) {
    CUDA_TRY(cudaEventSynchronize(ev[n]));
    for (int i = 0; i < n; ++i) {
      float ms = 0;
      CUDA_TRY(cudaEventElapsedTime(&ms, ev[i], ev[i + 1]));
      acc[i] += ms;
    }
  }
  for (int i = 0; i < n; ++i) layer_ms[i] = (float)acc[i];
  if (n_steps) *n_steps = (int)net->timing_sets.size();
  for (auto &ev : net->timing_sets) net->timing_free.push_back(std::move(ev));
  net->timing_sets.clear();
  return PCNN_OK;
}

pcnn_status pcnn_last_launch_count(const pcnn_net *net, int *launches) {
  if (!net || !launches) return fail(PCNN_ERR_INVALID_ARGUMENT, "null argument");
  *launches = net->launches_per_infer;
  return PCNN_OK;
}

// Debug export (not part of include/pcnn.h): tcgen05 kernel role-wait counters.
pcnn_status pcnn_debug_tc_profile(int reset, unsigned long long out[32]) {
  CUDA_TRY(tc_profile(reset, out));
  return PCNN_OK;
}

// Debug export: FC kernel timeline counters (prof build)
pcnn_status pcnn_debug_fc_profile(int reset, unsigned long long out[16]) {
  CUDA_TRY(fc_profile(reset, out));
  return PCNN_OK;
}

pcnn_status pcnn_enable_sm_census(pcnn_net *net, int enable) {
  if (!net) return fail(PCNN_ERR_INVALID_ARGUMENT, "null net");
  net->census = enable != 0;
  net->version++;
  return PCNN_OK;
}

pcnn_status pcnn_get_sm_census(pcnn_net *net, int layer, unsigned int mask_out[8]) {
  if (!net || !mask_out || layer < 0 || layer >= (int)net->layers.size())
    return fail(PCNN_ERR_INVALID_ARGUMENT, "bad arguments");
  CUDA_TRY(cudaSetDevice(net->device));
  CUDA_TRY(cudaMemcpy(mask_out, net->layers[layer].d_census, 32, cudaMemcpyDeviceToHost));
  return PCNN_OK;
}

}  // extern "C"
