/*
 * pcnn.h -- C ABI of the B200-native P-CNN batched-inference hot path.
 *
 * The operations are the ones PAPER.md (Song et al., HPCA'17) states as the
 * problem (cited P:<line>):
 *   - deploy a trained CNN without retraining
 *   - execute inference: conv = im2col + GEMM (F_m x D_m)       P:53-61, Fig. 2
 *     max-pooling and classifier layers
 *     output probabilities and their entropy (eq. 2)
 *   - choose per layer a faster, less precise kernel variant
 *     (here: rank-r factorisation, north_star; R7)
 *   - give each layer optSM SMs x optTLP CTAs
 *
 * Conventions for every function:
 *   - Returns a pcnn_status; nothing throws across the ABI.  On failure a
 *     thread-local message is available from pcnn_last_error_message().
 *   - Layer indices are 0-based positions in the descriptor list.
 *   - "host" pointers are ordinary CPU memory; "device" pointers are CUDA
 *     device memory on the net's device.  The caller keeps ownership of every
 *     pointer it passes; host weight/bias arrays are read during the call and
 *     never retained.  The library owns packed weights, factor caches, the
 *     activation arena and its CUDA graphs, all released by pcnn_destroy_net.
 *   - Streams are passed as `void*` holding a cudaStream_t (NULL = legacy
 *     default stream), so this header needs no CUDA headers.
 *   - Argument and shape errors are reported synchronously, before anything
 *     is enqueued.  Kernel launch failures return PCNN_ERR_CUDA; device faults
 *     surface at the caller's next synchronisation (CUDA convention).
 *   - A net is not re-entrant: at most one pcnn_infer* in flight per net, and
 *     pcnn_set_* must not be called while one is in flight.
 *   - There is no CPU fallback: every compute step runs in the library's CUDA
 *     kernels for sm_100a; without a usable B200 pcnn_create_net fails with
 *     PCNN_ERR_CUDA.
 */
#ifndef PCNN_H
#define PCNN_H

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
    PCNN_OK = 0,
    PCNN_ERR_INVALID_ARGUMENT = 1,
    PCNN_ERR_SHAPE = 2,
    PCNN_ERR_UNSUPPORTED = 3,
    PCNN_ERR_OUT_OF_MEMORY = 4,
    PCNN_ERR_CUDA = 5,
    PCNN_ERR_BATCH_TOO_LARGE = 6
} pcnn_status;

typedef enum {
    PCNN_CONV = 0,     /* conv + bias (+ReLU): Fig. 2             */
    PCNN_LRN = 1,      /* across-channel LRN (Caffe; R3)          */
    PCNN_MAXPOOL = 2,  /* max pooling, no padding (R4)                */
    PCNN_AVGPOOL = 3,  /* average pooling, no padding (R4)                  */
    PCNN_FC = 4        /* classifier layer y = Wx + b (+ReLU) (R5)    */
} pcnn_layer_kind;

typedef enum {
    PCNN_FP32_SIMT = 0, /* FP32 FFMA check path (the paper's SGEMM)  */
    PCNN_TF32 = 1,      /* tcgen05 kind::tf32, operands RN-rounded (R9)     */
    PCNN_BF16 = 2       /* tcgen05 kind::f16 with BF16 operands (R9)        */
} pcnn_precision;

typedef enum {
    PCNN_VARIANT_EXACT = 0, /* the exact layer                              */
    PCNN_VARIANT_RANK = 1   /* rank-r two-stage factorisation (R7)          */
} pcnn_variant;

/* One layer.  Unused fields are ignored for a kind.
 *   CONV  : out_channels = N_f, kernel = S_f, stride, pad, groups (Caffe
 *           groups: N_f and the input channels must be divisible), relu.
 *   FC    : out_channels = output features, relu.  Input is the previous
 *           activation flattened in C,H,W order (R5).
 *   LRN   : kernel = local size n (odd), lrn_alpha, lrn_beta, lrn_k.
 *   POOLS : kernel = window k, stride. */
typedef struct {
    int kind;
    int out_channels;
    int kernel;
    int stride;
    int pad;
    int groups;
    int relu;
    float lrn_alpha;
    float lrn_beta;
    float lrn_k;
} pcnn_layer_desc;

/* Layout choices of pcnn_create_net (pcnn_net_desc.flags, OR-ed).  Every
 * combination computes the same layers (the same products per output, up to
 * the accumulation order and last-place rounding of fused epilogues, bounded
 * in DESIGN.md); 0 = the library's default plan.  They exist so that tests
 * can compare the alternative kernels / layouts against each other. */
typedef enum {
    PCNN_FLAG_NO_SPACE_TO_DEPTH = 1,    /* strided / 3-channel first conv read
                                           from a channel-padded input
                                           instead of space-to-depth or
                                           im2col staging (a1)               */
    PCNN_FLAG_NO_PADDED_LAYOUT = 2,     /* every conv in TMA-im2col mode (no
                                           zero-haloed shifted windows)      */
    PCNN_FLAG_NO_LRN_POOL_FUSION = 4,   /* LRN and the following pool as two
                                           launches (and no conv+LRN epilogue) */
    PCNN_FLAG_CONV_LRN_EPILOGUE = 8,    /* conv -> LRN fused into the tcgen05
                                           epilogue also for padded-layout
                                           convs (off by default: slower)    */
    PCNN_FLAG_NARROW_SLABS = 16,        /* grouped convs with channels per
                                           group not a multiple of 128 B keep
                                           them unpadded (SW64 / SW32 slabs) */
    PCNN_FLAG_PERFORATION_IM2COL = 32,  /* row perforation of padded-layout
                                           layers in im2col mode (NEXT-1)    */
    PCNN_FLAG_PER_ROW_WINDOWS = 64      /* padded-layout convs load one A
                                           window per filter row (never one
                                           whole-slab window for all taps)   */
} pcnn_net_flag;

typedef struct {
    int in_channels;   /* C of the NCHW input images                        */
    int in_height;     /* H                                                  */
    int in_width;      /* W                                                  */
    int max_batch;     /* largest batch pcnn_infer* will be called with      */
    int precision;     /* pcnn_precision                                     */
    int device;        /* CUDA device ordinal                                */
    int flags;         /* OR of pcnn_net_flag, 0 = default                   */
} pcnn_net_desc;

/* Per-layer geometry / plan, for a given batch (pcnn_query_layer,
 * pcnn_describe_net).  GEMM dims are per group (eq. 4 M x N, K). */
typedef struct {
    int kind;
    int in_c, in_h, in_w;
    int out_c, out_h, out_w;
    int groups;
    long long gemm_m;   /* B * H_o * W_o (GEMM rows = output pixels)         */
    int gemm_n;         /* N_f / g                                           */
    int gemm_k;         /* S_f^2 * C / g                                     */
    double flops;       /* algorithmic FLOPs of the active variant (eq. 1)  */
    double flops_exact; /* eq. 1 FLOPs of the exact layer                    */
    double bytes;       /* algorithmic bytes: in + out activations at storage
                           precision + weights once                          */
    int variant;        /* pcnn_variant in effect                            */
    int rank;           /* r when variant == RANK, else 0                    */
    int n_sms;          /* SM budget in effect (0 = all)                     */
    int tlp;            /* CTAs per SM in effect                             */
    int engine;         /* 0 = SIMT kernel, 1 = tcgen05 kernel, 2 = no GEMM  */
    int tile_m, tile_n; /* GEMM tile (sub-matrix m x n)               */
    long long tiles;    /* GridSize, eq. 4 (all groups)                      */
    int grid;           /* CTAs launched                                     */
    double util;        /* eq. 6 with maxBlocks = n_sms * tlp                */
    double rec;         /* eq. 9 (tile-padding efficiency)                   */
    int splits;         /* split-K factor of the GEMM (1 = none)             */
    int a_mode;         /* tcgen05 A-operand addressing: 0 = TMA im2col over
                           output pixels, 1 = rectangle tiles (opt-in),
                           2 = padded-layout shifted window (one TMA row
                           window per filter row feeds all S taps),
                           3 = FC weight stream (tile_m = weight rows per
                           CTA, tile_n = images per UMMA, splits = K split
                           of a CTA cluster)                                 */
    int halo_in, halo_out; /* zero border of the stored input / output
                           activation layouts ([B][H+2h][W+2h][C])           */
    int cta_group;      /* SMs per GEMM tile: 2 for CTA-pair tiles, else 1   */
    double t_unit_us;   /* modelled time of one work unit (tile, or one split
                           of an FC unit) on its cta_group SMs (eq. 12 per
                           wave); non-GEMM layers: 0                          */
    int whole_window;   /* a_mode 2 only: 1 = one TMA window of 128 + (S-1) x
                           (grid width + 1) rows per channel slab feeds all
                           S x S taps (fewer A bytes for narrow grids), 0 =
                           one window per filter row                          */
} pcnn_layer_info;

/* Resource + time model of one layer, for the
 * layer's current variant at `batch`, on the whole device:
 *   grid_size     GridSize = work units of the layer's GEMM (eq. 4 tiles x
 *                 split-K factor); non-GEMM layers: 0
 *   opt_tlp       CTAs per SM: 1 for tcgen05 kernels (one CTA per SM by
 *                 shared memory / TMEM), the kernel's occupancy for SIMT
 *   n_invocations eq. 8 on all SMs: ceil(GridSize / (TLP * nSMs)), with
 *                 nSMs counted in CTA-pair units for 2-SM tiles
 *   opt_sm        eq. 11: the fewest SMs that keep n_invocations (a
 *                 multiple of cta_group); all SMs for non-GEMM layers
 *   t_model_us    eq. 12 at opt_sm (R12 / NEXT-3): t = t_launch +
 *                 n_invocations x t_unit, where t_unit = FLOPs per work unit
 *                 / (peak per SM x pipe efficiency), bounded below by the
 *                 unit's operand bytes at the measured L2->SM rate (eq. 12's
 *                 rEC enters through the padded tile), and t_launch the
 *                 measured fixed cost of one launch (launch, prologue, pipe
 *                 fill, epilogue drain); non-GEMM layers: t_launch + their
 *                 algorithmic bytes at min(HBM, n x per-SM) bandwidth
 *   t_launch_us   the fixed term above
 *   t_unit_us     the per-wave term above
 * Host-only (no launch); INVALID_ARGUMENT for a bad layer / batch. */
typedef struct {
    long long grid_size;
    int opt_tlp;
    int n_invocations;
    int opt_sm;
    int cta_group;
    double t_model_us;
    double t_launch_us;
    double t_unit_us;
} pcnn_budget_plan;

typedef struct pcnn_net pcnn_net;

/* Build a net: validate descriptors, infer shapes, pack weights into the
 * kernel layouts (K-major, NHWC order, precision-rounded), allocate the
 * activation arena for max_batch and plan every layer.
 *   weights[i] : host fp32; CONV in OIHW [N_f][C/g][S][S], FC in
 *                [out][in] with `in` in C,H,W order; NULL for weightless kinds.
 *   biases[i]  : host fp32 [out_channels]; NULL = zero bias.
 * Errors: INVALID_ARGUMENT / SHAPE / UNSUPPORTED (a layer shape the kernels
 * cannot take), OUT_OF_MEMORY, CUDA (no device / not sm_100). */
pcnn_status pcnn_create_net(const pcnn_net_desc *desc,
                            const pcnn_layer_desc *layers, int n_layers,
                            const float *const *weights,
                            const float *const *biases, pcnn_net **out);

pcnn_status pcnn_destroy_net(pcnn_net *net);

/* Select a layer's variant (P:335 accuracy tuning picks, P:345 calibration
 * backtracks).  RANK: rank in [1, min(N_f/g, S^2 C/g)]; the library computes a
 * truncated SVD of each group's F_m on the host (FP64 one-sided Jacobi) the
 * first time, caches it, and runs stage 1 (S x S conv, r filters) then stage 2
 * (1x1, r -> N_f/g, + bias + ReLU).  rank == min(...) is full rank.
 * EXACT ignores `rank`.  Errors: UNSUPPORTED for LRN / pool layers,
 * INVALID_ARGUMENT for a bad rank. */
pcnn_status pcnn_set_variant(pcnn_net *net, int layer, int variant, int rank);

/* Perforation-interpolation variant (Fig. 11; reading
 * R13): the conv is evaluated only at the kept positions of an sh x sw
 * output grid (rows 0, sh, 2sh, ...; columns 0, sw, ...) -- perforation rate
 * 1 - H'W'/(HW) -- and every other output position takes the value of its
 * nearest kept neighbour (ties to the lower index).  sh = sw = 1 turns it off;
 * steps 1..4.  Conv layers on the tcgen05 engine (BF16 / TF32) only;
 * UNSUPPORTED for the FP32 SIMT path, a staged first conv, or a layer with a
 * rank variant (pcnn_set_variant(EXACT) clears both). */
pcnn_status pcnn_set_perforation(pcnn_net *net, int layer, int sh, int sw);

/* Install explicit factors for a RANK variant (conv: test hook; FC: the way
 * to get an FC rank-r variant -- the library computes SVDs only for conv
 * layers, whose per-group matrices are small).
 *   conv: A host fp32 [groups][N_f/g][rank]   (stage-2 1x1 weights)
 *         B host fp32 [groups][rank][C/g][S][S] (stage-1 filters, OIHW)
 *         -> conv(x, A_g B_g) + bias
 *   FC:   A host fp32 [N][rank], B host fp32 [rank][C*H*W] (columns in the
 *         input's C,H,W order like the FC weight) -> (A B) x + bias
 * INVALID_ARGUMENT for a rank outside [1, min(N, K)]; UNSUPPORTED for other
 * layer kinds or a perforated layer. */
pcnn_status pcnn_set_variant_factors(pcnn_net *net, int layer, int rank,
                                     const float *A, const float *B);

/* Per-layer SM / CTA budget (P:213 PSM, P:341 optSM x optTLP): the layer's
 * kernels run on at most n_sms SMs with at most ctas_per_sm CTAs each.
 * n_sms = 0 means all SMs; values above the device count are clamped.
 * ctas_per_sm = 0 means the kernel's natural occupancy.  tcgen05 kernels are
 * 1 CTA/SM by construction (their tlp is reported as 1).  Floors: a CTA-pair
 * conv tile needs 2 SMs, an FC layer 2 x splits SMs (its K split is one
 * co-resident group of CTA pairs; pcnn_query_layer reports splits).  The budget changes
 * placement only: results are bitwise identical for every budget (R11). */
pcnn_status pcnn_set_sm_budget(pcnn_net *net, int layer, int n_sms,
                               int ctas_per_sm);

/* Per-layer tile choice override (the paper's sub-matrix choice, P:186,
 * P:223, eqs. 4-9): cta_group = 1 (128-row UMMA tiles) or 2
 * (CTA-pair 256-row tiles), m_sub = 128-row M sub-tiles per CTA sharing each
 * weight slab in padded-layout mode (1 or 2); 0 = the planner's choice.  The
 * K order of every output is unchanged, so results are bitwise identical to
 * the default plan's.  UNSUPPORTED for non-GEMM layers or the FP32 SIMT
 * engine, INVALID_ARGUMENT for other values. */
pcnn_status pcnn_set_layer_plan(pcnn_net *net, int layer, int cta_group,
                                int m_sub);

/* The hot path.  Asynchronous on `stream`.
 *   d_images  : device fp32 [batch][C][H][W] (NCHW)
 *   d_out     : device fp32 [batch][pcnn_output_size()] -- the last layer's
 *               output flattened in C,H,W order (logits for a classifier)
 *   d_probs   : device fp32 [batch][pcnn_output_size()] softmax, or NULL
 *   d_entropy : device fp32 [batch] entropy (eq. 2, natural log), or NULL
 * 1 <= batch <= max_batch (else BATCH_TOO_LARGE / INVALID_ARGUMENT).  The
 * launch sequence is captured once per (batch, pointers, variant/budget
 * state) into a CUDA graph and replayed. */
pcnn_status pcnn_infer(pcnn_net *net, const float *d_images, int batch,
                       float *d_out, float *d_probs, float *d_entropy,
                       void *stream);

/* End-to-end form of pcnn_infer with HOST buffers: copies h_images to a
 * library-owned device buffer, runs the hot path, copies the outputs back and
 * synchronises `stream` before returning.  Host buffers should be pinned for
 * full PCIe bandwidth.  h_probs / h_entropy may be NULL.  When the images take
 * much longer to copy than to infer (batch >= 64 and the copy per image > 2x
 * the modelled compute per image, e.g. AlexNet), the batch runs as 4 chunks
 * whose host->device copies (on a library stream) overlap the previous
 * chunk's inference.  Per-image results are bitwise those of pcnn_infer on
 * the whole batch (the FC K split is batch-independent; conv layers split K
 * only when their tiles cannot fill the device, which no chunk >= 16 images
 * of AlexNet / VGG-16 reaches). */
pcnn_status pcnn_infer_host(pcnn_net *net, const float *h_images, int batch,
                            float *h_out, float *h_probs, float *h_entropy,
                            void *stream);

/* pcnn_infer_host for 8-bit images, the pixels' native format: h_pixels
 * [batch][C][H][W] uint8 (host, pinned for full PCIe bandwidth).  The network
 * input is x = (pixel - mean[c]) * scale (mean: C floats, NULL = 0), computed
 * on the device (exact for integer pixels and mean, scale 1); everything else
 * as pcnn_infer_host -- PCIe carries 1 B per pixel instead of 4.  The batch
 * runs as 4 pipelined chunks when the copy per image exceeds a quarter of
 * the modelled compute per image.  Per-image results are bitwise those of
 * pcnn_infer on the converted images. */
pcnn_status pcnn_infer_host_u8(pcnn_net *net, const unsigned char *h_pixels,
                               const float *mean, float scale, int batch,
                               float *h_out, float *h_probs, float *h_entropy,
                               void *stream);

/* Elements per image of d_out (C*H*W of the last layer). */
pcnn_status pcnn_output_size(const pcnn_net *net, int *out_elems);

/* Number of layers and the plan of one layer for `batch` images. */
pcnn_status pcnn_num_layers(const pcnn_net *net, int *n_layers);
pcnn_status pcnn_query_layer(const pcnn_net *net, int layer, int batch,
                             pcnn_layer_info *info);
/* eqs. 8 / 11 / 12 for one layer (pcnn_budget_plan above). */
pcnn_status pcnn_plan_budget(const pcnn_net *net, int layer, int batch,
                             pcnn_budget_plan *plan);

/* eq. 12 time model of one layer at `batch` on n_sms SMs (0 = all), the
 * same terms as pcnn_budget_plan: t_launch + n_invocations(n_sms) x t_unit,
 * with n_invocations from eq. 8 at that budget.  Host-only. */
pcnn_status pcnn_model_layer_time(const pcnn_net *net, int layer, int batch,
                                  int n_sms, double *t_us);

/* Host-only shape inference + FLOP/byte accounting of a descriptor list,
 * no device needed (used by CPU tests and by planners).  infos[n_layers]. */
pcnn_status pcnn_describe_net(const pcnn_net_desc *desc,
                              const pcnn_layer_desc *layers, int n_layers,
                              int batch, pcnn_layer_info *infos);

/* Per-layer latency: run the net `reps` times (not graph-captured) with CUDA
 * events around every layer on `stream`; layer_ms[n_layers] receives the mean
 * milliseconds per layer, *total_ms (nullable) the mean whole pass (staging
 * and softmax included).  Synchronises `stream`. */
pcnn_status pcnn_profile_layers(pcnn_net *net, const float *d_images,
                                int batch, float *d_out, int reps,
                                float *layer_ms, float *total_ms,
                                void *stream);

/* Live per-layer timing.  While enabled, pcnn_infer runs without CUDA graphs
 * and records a CUDA event on the caller's stream after input staging and
 * after every layer.  pcnn_read_layer_timing synchronises those events and
 * returns, per layer, the milliseconds summed over all pcnn_infer calls since
 * the previous read (*n_steps = number of calls), then resets. */
pcnn_status pcnn_set_layer_timing(pcnn_net *net, int enable);
pcnn_status pcnn_read_layer_timing(pcnn_net *net, float *layer_ms,
                                   int *n_steps);

/* Number of CUDA kernels the last pcnn_infer enqueue launched (a graph
 * replay launches the same kernels as the capture that built it). */
pcnn_status pcnn_last_launch_count(const pcnn_net *net, int *launches);

/* Test hook: when enabled, every admitted CTA of every layer kernel records
 * its %smid; pcnn_get_sm_census returns the 256-bit SM mask (8 words) seen
 * by `layer` during the last pcnn_infer.  Disabling frees the buffers. */
pcnn_status pcnn_enable_sm_census(pcnn_net *net, int enable);
pcnn_status pcnn_get_sm_census(pcnn_net *net, int layer,
                               unsigned int mask_out[8]);

/* Number of SMs of `device` (0 if none), and the library's version string. */
int pcnn_device_sm_count(int device);
const char *pcnn_version(void);

const char *pcnn_status_string(pcnn_status status);
const char *pcnn_last_error_message(void);

#ifdef __cplusplus
}
#endif
#endif /* PCNN_H */
