// kernels_tc.cu -- tcgen05 implicit-GEMM convolution / FC for sm_100a (K1/K2).
//
// What it computes (Fig. 2; eq. 1): for every group g,
//   O_g[M x Nfg] = im2col(X)_g[M x K] * F_m,g[Nfg x K]^T  (+bias, ReLU)
// with M = B*Ho*Wo output pixels (NHWC rows), K = (r, s, c) taps x channels.
// D_m (the im2col matrix) is never materialised: the A tile of every K-block
// is fetched by TMA in im2col mode -- 128 consecutive output pixels x one
// filter tap (r, s) x a channel slab, with conv padding and ragged tails
// zero-filled by the TMA unit -- straight into the swizzled shared-memory
// layout the UMMA descriptor expects.  A K-block is 128 B of K per row: one
// 64-channel slab (SW128), or 2 / 4 narrower slabs (SW64 / SW32) when the
// channels per group are not a multiple of 64 (AlexNet conv2: 48).  The
// weight tile (B operand) arrives by a tiled TMA load.  One thread issues all
// loads, one thread issues tcgen05.mma (BF16 kind::f16 or kind::tf32, FP32
// accumulate) into a double-buffered TMEM accumulator, and four epilogue
// warps drain it with tcgen05.ld, add bias, apply ReLU, round to the storage
// precision and store NHWC rows (or, for split-K work units, FP32 partial
// sums that a deterministic reduction kernel adds in split order).
// The kernel is persistent: grid = min(work units, SM budget) CTAs, 1 CTA per
// SM (smem + TMEM), static round-robin schedule -- the grid cap IS the
// per-layer SM budget.  The pipeline depth is sized at launch from
// the N tile (~200 KB of operand stages per SM).
//
// CG = 2 runs the same pipeline on a CTA pair (cluster of 2, cta_group::2):
// one 256 x N tile per pair, each CTA loading its 128 A rows and half of the
// weight tile into its own smem with the loads' bytes counted on the leader's
// barrier; the leader issues M = 256 UMMAs whose accumulator rows are split
// across both CTAs' TMEM, and its commits multicast to both CTAs' barriers.
//
// CTA = 6 warps: warp 0 TMA producer, warp 1 TMEM allocator + MMA issuer,
// warps 2..5 epilogue (TMEM lane quarter = warp % 4).
#include <algorithm>
#include <cstdlib>

#include "budget.cuh"
#include "lrn_math.cuh"
#include "pcnn_internal.h"
#include "tc_ptx.cuh"

namespace pcnn {

constexpr int TC_BM = 128;              // UMMA M (cta_group::1)
constexpr int TC_BN_MAX = 256;          // max UMMA N
constexpr int TC_ROW_BYTES = 128;       // one K-block row = one 128B swizzle row
constexpr int TC_MAX_STAGES = 12;
constexpr int TC_MAX_BSTAGES = 24;      // padded mode with narrow (SW64/SW32) slabs
constexpr int TC_A_STAGE = TC_BM * TC_ROW_BYTES;          // 16 KB
constexpr int TC_STAGE_BUDGET = 176 * 1024;               // operand stages per CTA
constexpr int TC_MAX_KTAB = 1024;       // slab-table entries kept in smem
constexpr int EPI_PITCH = 144;          // epilogue staging row: 128 B + 16 B pad
// per-warp staging slot: 32 rows x 144 B (st.global path) or one 32-row x
// 32-column swizzled TMA-store box (<= 4 KB); 1024-aligned slots
constexpr int EPI_WARP_BYTES = 5120;
// warps: 0 TMA producer, 1 MMA issuer, then NEPI = 8 epilogue warps (two per
// TMEM lane quarter splitting the columns, also in the LRN-fused variant)
template <bool LRN> __host__ __device__ constexpr int tc_nepi() { return 8; }
template <bool LRN> __host__ __device__ constexpr int tc_threads() { return 64 + 32 * tc_nepi<LRN>(); }
constexpr int TC_TMEM_COLS = 512;       // 2 accumulator buffers x 256 columns

// smem layout (bytes from the 1024-aligned base):
//   [0, TC_STAGE_BUDGET)   A stages, then B stages (runtime count)
//   SM_EPI                 per-epilogue-warp output staging (8 warps, 1024-aligned)
//   SM_BAR                 barriers + TMEM pointer
//   SM_KTAB                (r, s, c) table, one entry per A slab
constexpr int SM_EPI = TC_STAGE_BUDGET;
constexpr int SM_BAR = SM_EPI + 8 * EPI_WARP_BYTES;
constexpr int SM_FULL = SM_BAR;
constexpr int SM_EMPTY = SM_FULL + 8 * TC_MAX_BSTAGES;
constexpr int TC_MAX_TBUF = 8;         // TMEM accumulator buffers (narrow N tiles)
constexpr int SM_TFULL = SM_EMPTY + 8 * TC_MAX_BSTAGES;
constexpr int SM_TEMPTY = SM_TFULL + 8 * TC_MAX_TBUF;
constexpr int SM_TMEMPTR = SM_TEMPTY + 8 * TC_MAX_TBUF;
constexpr int TC_MAX_ASTAGES = 8;       // padded mode: A row-window ring
constexpr int SM_AFULL = SM_TMEMPTR + 16;
constexpr int SM_AEMPTY = SM_AFULL + 8 * TC_MAX_ASTAGES;
constexpr int SM_KTAB = SM_BAR + 1024;
static_assert(SM_AEMPTY + 8 * TC_MAX_ASTAGES <= SM_KTAB, "barrier area");
constexpr int SM_TOTAL = SM_KTAB + 4 * TC_MAX_KTAB;
constexpr size_t TC_SMEM_BYTES = SM_TOTAL + 1024;         // + alignment slack

size_t tc_smem_bytes() { return TC_SMEM_BYTES; }
int tc_max_ktab() { return TC_MAX_KTAB; }
int tc_block_k_elems(int st) { return st == ST_BF16 ? 64 : 32; }
// Padded mode: one A stage is the (128 + 2 pad)-row window of one filter row
// r and channel slab (msub = 2: two such windows, 128 rows apart, for two
// M sub-tiles that share every weight slab); one B stage is the weight slab
// of one tap (r, s).
// rows from one sub-tile's window to the next: a whole number of 8-row
// swizzle atoms, so every window starts swizzle-aligned
__host__ __device__ constexpr int pm_sub_rows(int S) { return (TC_BM + S - 1 + 7) / 8 * 8; }
// A window rows per sub-tile: per filter row (ww = 0) or whole (ww = 1)
int pm_window_rows(int S, int wv, int ww) { return ww ? TC_BM + (S - 1) * (wv + 1) : TC_BM + S - 1; }
static int pm_a_stage_bytes(int slab_bytes, int rows, int msub) {
  const int sub = (rows + 7) / 8 * 8;
  return ((msub - 1) * sub * slab_bytes + rows * slab_bytes + 1023) / 1024 * 1024;
}
void tc_pm_stages(int bn, int cg, int slab_bytes, int S, int msub, int *a_stages, int *b_stages,
                  int rows, int ww) {
  const int as_bytes = pm_a_stage_bytes(slab_bytes, rows, msub);
  const int bs_bytes = bn / cg * slab_bytes;
  // 128 B slabs keep the tuned ring depths (4 windows, 12 tap slabs); narrow
  // slabs carry 2-4x less work per stage and get deeper rings.  Whole windows
  // keep >= 8 tap slabs in flight (a window's S*S slabs stream through them).
  int na = slab_bytes == 128 ? 4 : TC_MAX_ASTAGES;
  const int bmin = ww ? 6 : 2 * S;
  while (na > 2 && na * as_bytes + bmin * bs_bytes > TC_STAGE_BUDGET) --na;
  int nb = (TC_STAGE_BUDGET - na * as_bytes) / bs_bytes;
  const int nb_max = slab_bytes == 128 && !ww ? TC_MAX_STAGES : TC_MAX_BSTAGES;
  if (nb > nb_max) nb = nb_max;
  *a_stages = na;
  *b_stages = nb;
}

int tc_stages_for(int bn, int cg) {
  const int per = TC_A_STAGE + bn / cg * TC_ROW_BYTES;
  int n = TC_STAGE_BUDGET / per;
  if (n > TC_MAX_STAGES) n = TC_MAX_STAGES;
  static const char *ov = exp_env("PCNN_STAGES");     // tuning experiments only
  if (ov && atoi(ov) >= 2 && atoi(ov) < n) n = atoi(ov);
  return n;
}

// Instruction descriptor: D fp32, A/B = BF16 (1) or TF32 (2), K-major,
// M = 128 * CG, N = bn.
template <int ST, int CG>
__device__ __forceinline__ uint32_t umma_idesc(int bn) {
  const uint32_t fmt = ST == ST_BF16 ? 1u : 2u;
  return (1u << 4) | (fmt << 7) | (fmt << 10) | ((uint32_t)(bn >> 3) << 17) |
         ((uint32_t)((TC_BM * CG) >> 4) << 24);
}

struct TcArgs {
  ConvGeom g;
  FastDiv fd_mt, fd_nt, fd_grp, fd_hw, fd_w;   // mtiles, ntiles, groups, hv*wv, wv
  void *y;
  float *ws;            // split-K partials [splits][M][out_cs] fp32 (splits > 1)
  const float *bias;
  const int *ktab;      // per-element (r,s,c) table (nullptr when S == 1)
  int bn;
  int mtiles, ntiles, splits, units;
  int kblocks, kb_per_split;
  int stages;
  int slab_bytes;       // 128 / 64 / 32: A K-block = 128 / slab_bytes TMA slabs
  // A addressing: rect_w == 0 -> TMA im2col over 128 consecutive output pixels;
  // rect_w > 0 -> the M tile is a rect_n x rect_h x rect_w block of output
  // pixels (<= 128) and each tap's A slab is one tiled 4-D TMA box at the
  // tap-shifted input corner (stride 1; padding = OOB zero fill)
  int rect_w, rect_h, rect_n;
  int rects_w, rects_h;  // rect grid per image: ceil(Wo / rect_w), ceil(Ho / rect_h)
  int prof;             // 1: accumulate per-role barrier-wait cycles (debug)
  int skip;             // debug: 1 skip A loads, 2 skip B loads, 4 skip MMAs
  int a_stages, b_stages, pm_a_stage;   // padded mode rings (g.pm)
  // padded mode, whole windows (ww = 1): ONE A window of pm_rows = 128 +
  // (S-1)(wv+1) rows per channel slab feeds all S x S taps (tap (r, s) = a
  // descriptor shift of r*wv + s rows) instead of one (128 + S - 1)-row
  // window per filter row; pm_sub = rows from one M sub-tile's window to the
  // next in the A stage (a whole number of 8-row swizzle atoms)
  int ww, pm_rows, pm_sub;
  int msub;             // padded mode: M sub-tiles of 128 rows per CTA sharing each B slab
  // TMEM accumulator ring: nbuf buffers of tbw columns (512 / tbw), sub-tile
  // sb at column tsub * sb of its buffer.  Narrow tiles get up to 8 buffers,
  // so the MMA runs several tiles ahead of a latency-bound epilogue.
  int nbuf, tbw, tsub;
  int kmma_last;        // padded mode: UMMAs (32 B of K each) of the last channel slab that
                        // touch real channels; the rest multiply zero padding and are skipped
  int lrn;              // 1: fused across-channel LRN (size 5) in the epilogue
  int tma_y;            // 1: full 32-column output chunks leave by TMA tensor store
  int tma_y64;          // 1: bf16 output, full 64-column chunks use the 128 B-row map
  float lrn_a_over_n, lrn_beta, lrn_k;
  Budget b;
};

// Each lane of an epilogue warp owns one output row (pixel).  It parks the
// row's next 128 B (8 x 16 B pieces, `np` valid) in the warp's smem staging
// rows, then the warp writes them back row-contiguously: 8 lanes per 128 B
// line, 4 full lines per store instruction (instead of 32 scattered 16 B
// pieces).  `rowaddr` is each lane's destination for its piece 0 (nullptr
// when its row is out of range).
__device__ __forceinline__ void epi_store_rows(uint8_t *stage, const uint4 (&pc)[8], int np,
                                               char *rowaddr, int lane) {
  uint8_t *mine = stage + lane * EPI_PITCH;
#pragma unroll
  for (int j = 0; j < 8; ++j)
    if (j < np) *(uint4 *)(mine + 16 * j) = pc[j];
  __syncwarp();
#pragma unroll
  for (int it = 0; it < 8; ++it) {
    const int p = it * 32 + lane, r = p >> 3, j = p & 7;
    char *dst = (char *)__shfl_sync(0xffffffffu, (unsigned long long)rowaddr, r);
    if (dst != nullptr && j < np)
      *(uint4 *)(dst + 16 * j) = *(const uint4 *)(stage + r * EPI_PITCH + 16 * j);
  }
  __syncwarp();
}

// One 32-column epilogue step: bias (issued before the TMEM load so the
// latencies overlap), TMEM load of the lane's row, ReLU, halo rows zeroed.
__device__ __forceinline__ void epi_chunk32(const TcArgs &a, uint32_t taddr, int col, bool valid,
                                            float (&f)[32]) {
  const float4 *bp = (const float4 *)(a.bias + col);
  float4 bb[8];
#pragma unroll
  for (int q = 0; q < 8; ++q) bb[q] = __ldg(bp + q);
  {
    uint32_t v[32];
    tmem_ld32(taddr, v);
    tmem_ld_wait();
#pragma unroll
    for (int i = 0; i < 32; ++i) f[i] = __uint_as_float(v[i]);
  }
#pragma unroll
  for (int q = 0; q < 8; ++q) {
    f[4 * q] += bb[q].x;
    f[4 * q + 1] += bb[q].y;
    f[4 * q + 2] += bb[q].z;
    f[4 * q + 3] += bb[q].w;
  }
  if (a.g.relu)
#pragma unroll
    for (int i = 0; i < 32; ++i) f[i] = fmaxf(f[i], 0.f);
  if (!valid)
#pragma unroll
    for (int i = 0; i < 32; ++i) f[i] = 0.f;
}
__device__ __forceinline__ uint4 pack_bf16x8(const float *f) {
  uint4 pk;
  uint32_t *pw = (uint32_t *)&pk;
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    __nv_bfloat162 b2 = __floats2bfloat162_rn(f[2 * i], f[2 * i + 1]);
    pw[i] = *(uint32_t *)&b2;
  }
  return pk;
}

// Epilogue with the following LRN layer fused in (R3; Caffe size
// 5).  The tile holds every channel of its pixels (bn == Nfg <= 128, one N
// tile).  The two warps of a TMEM lane quarter split the channels in halves
// (16-aligned); each thread streams its pixel's half through 16-column TMEM
// loads, 8 channels (one 16 B bf16 piece) at a time, with the window's 2
// channels on either side taken from the neighbouring columns (the other
// half's at the boundary).  Per value: bias, ReLU, rounding to the storage
// precision -- the value the stand-alone conv would have stored -- then the
// stand-alone LRN kernels' arithmetic (squares by __fmul_rn, lrn_normalise),
// so the result is the one of conv -> store -> LRN.
template <int ST>
__device__ __forceinline__ void lrn_x16(const TcArgs &a, uint32_t taddr, int c0, bool valid,
                                        float (&f)[16]) {
  const ConvGeom &g = a.g;
  if (c0 >= g.Nfg) {                                   // past the channels: zero
#pragma unroll
    for (int i = 0; i < 16; ++i) f[i] = 0.f;
    return;
  }
  uint32_t v[16];
  tmem_ld16(taddr + c0, v);
  const float4 *bp = (const float4 *)(a.bias + c0);
  float4 bb[4];
#pragma unroll
  for (int q = 0; q < 4; ++q) bb[q] = __ldg(bp + q);
  tmem_ld_wait();
#pragma unroll
  for (int i = 0; i < 16; ++i) {
    const float b = i % 4 == 0 ? bb[i / 4].x : i % 4 == 1 ? bb[i / 4].y : i % 4 == 2 ? bb[i / 4].z : bb[i / 4].w;
    float x = __uint_as_float(v[i]) + b;
    if (g.relu) x = fmaxf(x, 0.f);
    if constexpr (ST == ST_BF16) x = __bfloat162float(__float2bfloat16_rn(x));
    else if (g.out_mode == OUT_F32_TF32) x = tf32_rna_tc(x);
    f[i] = (c0 + i < g.Nfg && valid) ? x : 0.f;        // halo rows are stored as zeros
  }
}

template <int ST>
__device__ __forceinline__ void epilogue_lrn(const TcArgs &a, uint32_t taddr, bool mok,
                                             bool valid, size_t orow, uint8_t *stage,
                                             int lane, int half) {
  const ConvGeom &g = a.g;
  const int C = g.Nfg;
  const int ch = ((C + 1) / 2 + 15) & ~15;             // channels per half (16-aligned)
  const int lo = half * ch, hi = min(C, lo + ch);
  if (lo >= hi) return;                                // warp-uniform
  constexpr int EB = ST == ST_BF16 ? 2 : 4;
  constexpr int PER = 16 / EB;                         // channels per 16 B piece
  float A[16], Bv[16];
  float l0 = 0.f, l1 = 0.f;                            // channels c - 2, c - 1
  if (lo > 0) {
    lrn_x16<ST>(a, taddr, lo - 16, valid, A);
    l0 = A[14];
    l1 = A[15];
  }
  lrn_x16<ST>(a, taddr, lo, valid, A);
  lrn_x16<ST>(a, taddr, lo + 16, valid, Bv);
  char *rowp = mok ? (char *)a.y + (orow + lo) * EB : nullptr;
  uint4 pc[8];
  // ch <= 64: at most 8 steps of 8 channels, unrolled so every register
  // index is static; BF16 flushes its 128 B row piece once, FP32 every 4 steps
#pragma unroll
  for (int p = 0; p < 8; ++p) {
    const int c = lo + 8 * p;
    if (c >= hi) break;                                // warp-uniform
    const bool odd = (p & 1) != 0;
    float w[12];
    w[0] = l0;
    w[1] = l1;
#pragma unroll
    for (int i = 0; i < 8; ++i) w[2 + i] = odd ? A[8 + i] : A[i];
    w[10] = odd ? Bv[0] : A[8];
    w[11] = odd ? Bv[1] : A[9];
    float sq[12];
#pragma unroll
    for (int i = 0; i < 12; ++i) sq[i] = __fmul_rn(w[i], w[i]);
    float o[8];
    lrn_normalise<ST == ST_BF16, 5, 8>(sq, w + 2, a.lrn_k, a.lrn_a_over_n, a.lrn_beta, o);
    if constexpr (ST == ST_BF16) {
      pc[p] = pack_bf16x8(o);
    } else {
      float t[8];
#pragma unroll
      for (int i = 0; i < 8; ++i) t[i] = g.out_mode == OUT_F32_TF32 ? tf32_rna_tc(o[i]) : o[i];
      pc[(2 * p) % 8] = make_uint4(__float_as_uint(t[0]), __float_as_uint(t[1]),
                                   __float_as_uint(t[2]), __float_as_uint(t[3]));
      pc[(2 * p + 1) % 8] = make_uint4(__float_as_uint(t[4]), __float_as_uint(t[5]),
                                       __float_as_uint(t[6]), __float_as_uint(t[7]));
    }
    l0 = w[8];
    l1 = w[9];
    if (odd) {                                         // next 16 columns
#pragma unroll
      for (int i = 0; i < 16; ++i) A[i] = Bv[i];
      lrn_x16<ST>(a, taddr, c + 24, valid, Bv);
    }
    const bool last = c + 8 >= hi;
    if constexpr (ST == ST_BF16) {
      if (p == 7 || last) {
        const int np = min(p + 1, (hi - lo + PER - 1) / PER);
        epi_store_rows(stage, pc, np, rowp, lane);
      }
    } else {
      if (p % 4 == 3 || last) {
        const int base = (p / 4) * 8;                  // pieces already stored
        const int np = min(2 * (p % 4 + 1), (hi - lo + PER - 1) / PER - base);
        epi_store_rows(stage, pc, np, rowp ? rowp + base * 16 : nullptr, lane);
      }
    }
  }
}

// Debug counters (PCNN_TC_PROFILE=1): summed clock64 cycles per role.
//  0 producer waits on EMPTY   1 MMA waits on FULL   2 MMA waits on TEMPTY
//  3 epilogue waits on TFULL   4 CTA lifetime        5 K-blocks issued
//  6 epilogue busy cycles      7 CTAs
//  16.. timeline (globaltimer ns, summed over CTAs): 16 setup + PDL wait,
//  17 wait -> first accumulator ready (epilogue warp 2), 18 wait -> epilogue
//  done, 19 wait -> exit, 20 CTAs, 21 ~min entry, 22 max exit, 23 ~min wait,
//  24 max wait
__device__ unsigned long long g_tc_prof[32];
__device__ __forceinline__ unsigned long long gtimer() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}

// Role profiling is compiled in only with -DPCNN_TC_PROF=1 (tools/tc_roles.py
// builds such a library): its clocks and 64-bit sums cost the issue loops
// uniform registers.
#ifndef PCNN_TC_PROF
#define PCNN_TC_PROF 0
#endif
#define TC_PROF(a) (PCNN_TC_PROF && (a).prof)

struct WaitClock {
  bool on;
  unsigned long long acc = 0;
  __device__ __forceinline__ void wait(uint32_t bar, uint32_t parity) {
    if (PCNN_TC_PROF && on) {
      const long long t0 = clock64();
      mbar_wait(bar, parity);
      acc += (unsigned long long)(clock64() - t0);
    } else {
      mbar_wait(bar, parity);
    }
  }
};

__device__ __forceinline__ void advance(uint32_t &stage, uint32_t &phase, int stages) {
  if (++stage == (uint32_t)stages) {
    stage = 0;
    phase ^= 1;
  }
}

// ------------------------------------------------------------ MMA issuers
// The issue loops are written so that every tcgen05.mma operand (descriptors,
// TMEM column, instruction descriptor, accumulate flag) is warp-uniform and
// derived from kernel parameters and uniform loop counters: ptxas then keeps
// them in uniform registers and a K-block's 4 UMMAs issue back to back.  A
// per-iteration R2UR round trip (what a lane-dependent branch in the loop
// causes) costs ~150 cycles per UMMA, more than an N = 64 UMMA executes in
// (tools/mma_rate_probe.cu).  K offsets inside a K-block are compile-time:
// the A K-block is 128 / SLAB slabs of TC_BM rows, each SLAB / 32 UMMAs deep.
template <int SLAB>
__device__ __forceinline__ constexpr uint32_t a_koff(int k) {
  return (uint32_t)((k / (SLAB / 32)) * (TC_BM * SLAB / 16) + 2 * (k % (SLAB / 32)));
}

template <int ST, int CG, int SLAB>
__device__ __forceinline__ void mma_issuer_im2col(const TcArgs &a, uint32_t sbase, uint32_t sA,
                                                  uint32_t sB, uint32_t b_stage,
                                                  uint32_t tmem_base, int pair, int npairs,
                                                  unsigned long long *acc_full,
                                                  unsigned long long *acc_temp) {
  const uint32_t idesc = umma_idesc<ST, CG>(a.bn);
  const uint64_t a_desc0 = umma_desc(sA, SLAB);
  const uint64_t b_desc0 = umma_desc_sw128(sB);
  const uint32_t a_stage16 = TC_A_STAGE / 16, b_stage16 = b_stage / 16;
  const int stages = a.stages, units = a.units, mtiles = a.mtiles, ntiles = a.ntiles;
  const int groups = a.g.groups, kblocks = a.kblocks, kbs = a.kb_per_split;
  const bool prof = TC_PROF(a) != 0, skip_mma = (a.skip & 4) != 0;
  const bool leader = elect_one();
  WaitClock wfull{prof}, wtemp{prof};
  uint32_t stage = 0, phase = 0, lt = 0;
  for (int u = pair; u < units; u += npairs, ++lt) {
    const int sp = u / (mtiles * ntiles * groups);
    const int k0 = sp * kbs, k1 = min(kblocks, k0 + kbs);
    const uint32_t buf = lt % a.nbuf, use = lt / a.nbuf;
    wtemp.wait(sbase + SM_TEMPTY + 8 * buf, (use & 1) ^ 1);
    tc_fence_after();
    const uint32_t dcol = tmem_base + buf * a.tbw;
    for (int kb = k0; kb < k1; ++kb) {
      wfull.wait(sbase + SM_FULL + 8 * stage, phase);
      tc_fence_after();
      const uint64_t ad = a_desc0 + stage * a_stage16;
      const uint64_t bd = b_desc0 + stage * b_stage16;
      if (leader) {
        if (!skip_mma) {
          tc_mma<ST, CG>(dcol, ad + a_koff<SLAB>(0), bd, idesc, kb > k0 ? 1u : 0u);
          tc_mma<ST, CG>(dcol, ad + a_koff<SLAB>(1), bd + 2, idesc, 1u);
          tc_mma<ST, CG>(dcol, ad + a_koff<SLAB>(2), bd + 4, idesc, 1u);
          tc_mma<ST, CG>(dcol, ad + a_koff<SLAB>(3), bd + 6, idesc, 1u);
        }
        tc_commit<CG>(sbase + SM_EMPTY + 8 * stage);
      }
      __syncwarp();
      if (++stage == (uint32_t)stages) {
        stage = 0;
        phase ^= 1;
      }
    }
    if (leader) tc_commit<CG>(sbase + SM_TFULL + 8 * buf);
    __syncwarp();
  }
  *acc_full = wfull.acc;
  *acc_temp = wtemp.acc;
}

// Padded mode: per (slab, filter row) A window, S taps; tap s reads the
// window shifted by s rows (SLAB / 16 descriptor units per row).
template <int ST, int CG, int SLAB, int MSUB>
__device__ __forceinline__ void mma_issuer_pm(const TcArgs &a, uint32_t sbase, uint32_t sA,
                                              uint32_t sBp, uint32_t pm_b_bytes,
                                              uint32_t tmem_base, int pair, int npairs, int nj,
                                              unsigned long long *acc_full,
                                              unsigned long long *acc_temp) {
  constexpr int KMMA = SLAB / 32;
  constexpr uint32_t ROW16 = SLAB / 16;
  const uint32_t idesc = umma_idesc<ST, CG>(a.bn);
  const uint64_t a_desc0 = umma_desc(sA, SLAB);
  const uint64_t b_desc0 = umma_desc(sBp, SLAB);
  const uint32_t a_st16 = (uint32_t)a.pm_a_stage / 16, b_st16 = pm_b_bytes / 16;
  const int a_stages = a.a_stages, b_stages = a.b_stages, units = a.units, S = a.g.S;
  const int ww = a.ww, taps = ww ? S * S : S, wv = a.g.wv;
  const int j_last = ww ? nj - 1 : nj - S, kmma_last = a.kmma_last;   // windows of the last channel slab
  // sub-tile 1's window starts pm_sub rows into the A stage
  const uint32_t sub16 = (uint32_t)a.pm_sub * ROW16;
  const bool prof = TC_PROF(a) != 0, skip_mma = (a.skip & 4) != 0;
  const bool leader = elect_one();
  WaitClock wfull{prof}, wtemp{prof};
  uint32_t as = 0, aph = 0, bs = 0, bph = 0, lt = 0;
  const int tiles_all = a.mtiles * a.ntiles * a.g.groups, kbs = a.kb_per_split;
  for (int u = pair; u < units; u += npairs, ++lt) {
    const uint32_t buf = lt % a.nbuf, use = lt / a.nbuf;
    // split-K over the windows (small batches only): windows [j0, j1)
    const int sp = u / tiles_all, j0 = sp * kbs, j1 = min(nj, j0 + kbs);
    wtemp.wait(sbase + SM_TEMPTY + 8 * buf, (use & 1) ^ 1);
    tc_fence_after();
    const uint32_t dcol = tmem_base + buf * a.tbw;
    for (int j = j0; j < j1; ++j) {
      wfull.wait(sbase + SM_AFULL + 8 * as, aph);
      const uint64_t ad = a_desc0 + as * a_st16;
      const int kk = j >= j_last ? kmma_last : KMMA;
      for (int t = 0, r = 0, s2 = 0; t < taps; ++t) {
        wfull.wait(sbase + SM_FULL + 8 * bs, bph);
        tc_fence_after();
        // tap (r, s2): the window shifted by r*wv + s2 rows (ww) or s2 rows
        const uint64_t aw = ad + (uint32_t)(r * wv + s2) * ROW16;
        const uint64_t bd = b_desc0 + bs * b_st16;
        if (leader) {
          if (!skip_mma) {
#pragma unroll
            for (int sb = 0; sb < MSUB; ++sb) {
              const uint64_t awb = aw + sb * sub16;
              const uint32_t dc = dcol + sb * a.tsub;
              tc_mma<ST, CG>(dc, awb, bd, idesc, (j > j0 || t > 0) ? 1u : 0u);
#pragma unroll
              for (int k = 1; k < KMMA; ++k)
                if (k < kk) tc_mma<ST, CG>(dc, awb + 2 * k, bd + 2 * k, idesc, 1u);
            }
          }
          tc_commit<CG>(sbase + SM_EMPTY + 8 * bs);
        }
        __syncwarp();
        if (++bs == (uint32_t)b_stages) {
          bs = 0;
          bph ^= 1;
        }
        if (++s2 == S) {
          s2 = 0;
          ++r;
        }
      }
      if (leader) tc_commit<CG>(sbase + SM_AEMPTY + 8 * as);
      __syncwarp();
      if (++as == (uint32_t)a_stages) {
        as = 0;
        aph ^= 1;
      }
    }
    if (leader) tc_commit<CG>(sbase + SM_TFULL + 8 * buf);
    __syncwarp();
  }
  *acc_full = wfull.acc;
  *acc_temp = wtemp.acc;
}

template <int ST, int CG, bool LRN>
__global__ void __launch_bounds__(tc_threads<LRN>(), 1) __maxnreg__(LRN ? 200 : 200)
conv_tc_kernel(const __grid_constant__ CUtensorMap tmap_w,
               const __grid_constant__ CUtensorMap tmap_x,
               const __grid_constant__ CUtensorMap tmap_y,
               const __grid_constant__ CUtensorMap tmap_y64, const TcArgs a) {
  extern __shared__ uint8_t smem_raw[];
  const unsigned long long tl_entry = TC_PROF(a) ? gtimer() : 0;
  uint8_t *smem = (uint8_t *)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
  const uint32_t sbase = smem_u32(smem);
  const int tid = threadIdx.x;
  // warp index through a lane-0 shuffle: provably warp-uniform, so the role
  // branches below keep their loop state in uniform registers
  const int warp = __shfl_sync(0xffffffffu, tid >> 5, 0), lane = tid & 31;
  constexpr int ESZ = ST == ST_BF16 ? 2 : 4;
  const ConvGeom &g = a.g;
  const int stages = a.stages;
  const uint32_t rank = CG == 2 ? cluster_ctarank() : 0;   // 0 = leader
  const int pair = blockIdx.x / CG, npairs = gridDim.x / CG;
  const int b_rows = a.bn / CG;                            // weight rows per CTA
  const uint32_t sA = sbase;                                     // A stages
  const uint32_t sB = sbase + (uint32_t)stages * TC_A_STAGE;     // B stages
  const uint32_t b_stage = (uint32_t)b_rows * TC_ROW_BYTES;
  const int slab_bytes = a.slab_bytes;
  const int nslab = TC_ROW_BYTES / slab_bytes;
  const int slab_elems = slab_bytes / ESZ;
  const bool rect = a.rect_w > 0;
  const int rect_rows = rect ? a.rect_w * a.rect_h * a.rect_n : TC_BM;   // A rows loaded
  const uint32_t a_bytes = (uint32_t)rect_rows * TC_ROW_BYTES;         // per stage

  uint32_t *ktab_s = (uint32_t *)(smem + SM_KTAB);
  const bool use_tab = a.ktab != nullptr;
  const int nent = g.Kpad / slab_elems;
  if (use_tab) {
    for (int i = tid; i < nent && i < TC_MAX_KTAB; i += tc_threads<LRN>()) {
      const int k = i * slab_elems;
      ktab_s[i] = k < g.K ? (uint32_t)__ldg(&a.ktab[k]) : 0xFF000000u;
    }
  }
  if (tid == 0) {
    for (int s = 0; s < (g.pm ? a.b_stages : stages); ++s) {   // b_stages <= TC_MAX_BSTAGES
      mbar_init(sbase + SM_FULL + 8 * s, 1);
      mbar_init(sbase + SM_EMPTY + 8 * s, 1);
    }
    for (int s = 0; s < (g.pm ? a.a_stages : 0); ++s) {
      mbar_init(sbase + SM_AFULL + 8 * s, 1);
      mbar_init(sbase + SM_AEMPTY + 8 * s, 1);
    }
    for (int i = 0; i < a.nbuf; ++i) {
      mbar_init(sbase + SM_TFULL + 8 * i, 1);
      mbar_init(sbase + SM_TEMPTY + 8 * i, tc_nepi<LRN>() * CG);   // one arrive per epilogue warp
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    census_mark(a.b);
  }
  if (warp == 1) {
    if constexpr (CG == 1) {
      asm volatile(
          "tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(
              sbase + SM_TMEMPTR),
          "n"(TC_TMEM_COLS));
      asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    } else {
      asm volatile(
          "tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(
              sbase + SM_TMEMPTR),
          "n"(TC_TMEM_COLS));
      asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;");
    }
  }
  tc_fence_before();
  if constexpr (CG == 2) cluster_sync(); else __syncthreads();
  tc_fence_after();
  const uint32_t tmem_base = *(volatile uint32_t *)(smem + SM_TMEMPTR);
  const int HoWo = g.Ho * g.Wo;
  // work unit u -> (m tile, n tile, group, split); m fastest so CTAs running
  // concurrently share one weight slice in L2.
  auto decode = [&](int u, int &mt, int &nt, int &grp, int &sp) {
    int r = (int)a.fd_mt.div((uint32_t)u);
    mt = u - r * a.mtiles;
    const int r2 = (int)a.fd_nt.div((uint32_t)r);
    nt = r - r2 * a.ntiles;
    sp = (int)a.fd_grp.div((uint32_t)r2);
    grp = r2 - sp * g.groups;
  };
  auto kb_range = [&](int sp, int &k0, int &k1) {
    k0 = sp * a.kb_per_split;
    k1 = min(a.kblocks, k0 + a.kb_per_split);
  };

  // L2 prefetch of the first unit's weight boxes: the weights do not depend on
  // the previous layer, so at small batches their first HBM touch overlaps its
  // tail (the A operand is read only after the PDL wait)
  if (warp == 0 && lane == 0 && pair < a.units) {
    int mt, nt, grp, sp;
    decode(pair, mt, nt, grp, sp);
    const int nrow = grp * g.Nfg + nt * a.bn + (int)rank * b_rows;
    if (g.pm) {
      const int pm_se0 = slab_bytes / ESZ, rw = a.ww ? g.S : 1;   // filter rows per window
      const int nj = (g.Cg / pm_se0) * g.S / rw;
      const int j0 = sp * a.kb_per_split, j1 = min(nj, j0 + a.kb_per_split);
      for (int j = j0, n = 0; j < j1 && n < 64; ++j) {
        const int cb = j * rw / g.S, r0 = j * rw - cb * g.S;
        for (int r = r0; r < r0 + rw; ++r)
          for (int s2 = 0; s2 < g.S; ++s2, ++n)
            tma_prefetch_2d(&tmap_w, (r * g.S + s2) * g.Cg + cb * pm_se0, nrow);
      }
    } else {
      int k0, k1;
      kb_range(sp, k0, k1);
      for (int kb = k0; kb < k1 && kb < k0 + 64; ++kb)
        tma_prefetch_2d(&tmap_w, kb * (TC_ROW_BYTES / ESZ), nrow);
    }
  }
  // PDL: setup above overlapped the previous kernel's tail; activations are
  // read (and outputs written) only after its completion
  pdl_enter();
  const long long t_start = TC_PROF(a) ? clock64() : 0;
  const unsigned long long tl_wait = TC_PROF(a) ? gtimer() : 0;
  unsigned long long tl_first = 0;
  unsigned long long wtf_acc_out = 0, busy_out = 0;   // epilogue profile (warp 2)

  // padded mode: K runs over (channel slab cb, filter row r) windows, each
  // feeding the S taps (r, s) of that row by shifting the A descriptor s rows
  const int pm_se = slab_bytes / ESZ;                  // channels per slab
  const int pm_nj = g.pm ? (g.Cg / pm_se) * (a.ww ? 1 : g.S) : 0;   // A windows per tile
  const uint32_t sBp = sbase + (uint32_t)a.a_stages * (uint32_t)a.pm_a_stage;
  const uint32_t pm_b_bytes = (uint32_t)b_rows * slab_bytes;
  if (warp == 0 && g.pm) {
    // ------------------------------------------------ TMA producer, padded mode
    if (lane == 0) {
      asm volatile("prefetch.tensormap [%0];" ::"l"((uint64_t)&tmap_w) : "memory");
      asm volatile("prefetch.tensormap [%0];" ::"l"((uint64_t)&tmap_x) : "memory");
      // pm = 2: nseg segments of wv + 2 pad columns (grid columns -pad ..)
      const uint32_t pm_a_bytes = g.pm == 2 ? (uint32_t)(g.nseg * (g.wv + 2 * g.pad)) * slab_bytes
                                            : (uint32_t)a.pm_rows * slab_bytes;
      uint32_t as = 0, aph = 0, bs = 0, bph = 0;
      WaitClock wc{TC_PROF(a) != 0};
      unsigned long long nkb = 0;
      for (int u = pair; u < a.units; u += npairs) {
        int mt, nt, grp, sp;
        decode(u, mt, nt, grp, sp);
        nkb += pm_nj;
        const int nrow = grp * g.Nfg + nt * a.bn + (int)rank * b_rows;
        const int i0 = (mt * CG + (int)rank) * TC_BM * a.msub;
        // split-K over the windows (small batches only): windows [j0, j1)
        const int j0 = sp * a.kb_per_split, j1 = min(pm_nj, j0 + a.kb_per_split);
        int cb = a.ww ? j0 : j0 / g.S, r = a.ww ? 0 : j0 - cb * g.S;
        for (int j = j0; j < j1; ++j) {
          wc.wait(sbase + SM_AEMPTY + 8 * as, aph ^ 1);
          const uint32_t fa = sbase + SM_AFULL + 8 * as;
          if (rank == 0) mbar_arrive_expect_tx(fa, (a.skip & 1) ? 0 : CG * a.msub * pm_a_bytes);
          if (!(a.skip & 1) && g.pm == 2) {
            // kept rows tb*nseg .. of image n, filter row r: a {slab, wv + 2 pad,
            // nseg} box starting pad columns left of the row, rows psh apart;
            // one box per M sub-tile
            const uint32_t dA = sA + as * (uint32_t)a.pm_a_stage;
            const int cc = grp * g.Cg + cb * pm_se;
            for (int sb = 0; sb < a.msub; ++sb) {
              const int T = (mt * CG + (int)rank) * a.msub + sb, n = T / g.tpi,
                        tb = T - n * g.tpi;
              const int grow = n * g.hv + g.vh + g.psh * tb * g.nseg + r - g.pad;
              tma_load_3d<CG>(dA + (uint32_t)(sb * a.pm_sub * slab_bytes), &tmap_x, fa,
                              cc, -g.pad, grow);
            }
          } else if (!(a.skip & 1)) {
            const uint32_t dA = sA + as * (uint32_t)a.pm_a_stage;
            const int cc = grp * g.Cg + cb * pm_se, row = i0 + (r - g.pad) * g.wv - g.pad;
            for (int sb = 0; sb < a.msub; ++sb) {
              const uint32_t d = dA + (uint32_t)(sb * a.pm_sub * slab_bytes);
              if constexpr (CG == 1) tma_load_2d(d, &tmap_x, fa, cc, row + sb * TC_BM);
              else tma_load_2d_2sm(d, &tmap_x, fa, cc, row + sb * TC_BM);
            }
          }
          advance(as, aph, a.a_stages);
          // the window's tap slabs: filter row r (per-row windows) or rows
          // 0 .. S-1 (whole windows), taps s2 = 0 .. S-1 of each
          for (int rr = r; rr < (a.ww ? g.S : r + 1); ++rr)
            for (int s2 = 0; s2 < g.S; ++s2) {
              wc.wait(sbase + SM_EMPTY + 8 * bs, bph ^ 1);
              const uint32_t fb = sbase + SM_FULL + 8 * bs;
              if (rank == 0) mbar_arrive_expect_tx(fb, (a.skip & 2) ? 0 : CG * pm_b_bytes);
              if (!(a.skip & 2)) {
                const int kk = (rr * g.S + s2) * g.Cg + cb * pm_se;
                if constexpr (CG == 1) tma_load_2d(sBp + bs * pm_b_bytes, &tmap_w, fb, kk, nrow);
                else tma_load_2d_2sm(sBp + bs * pm_b_bytes, &tmap_w, fb, kk, nrow);
              }
              advance(bs, bph, a.b_stages);
            }
          if (a.ww) ++cb;
          else if (++r == g.S) { r = 0; ++cb; }
        }
      }
      if (TC_PROF(a)) {
        atomicAdd(&g_tc_prof[0], wc.acc);
        atomicAdd(&g_tc_prof[5], nkb);
      }
    }
  } else if (warp == 1 && g.pm) {
    if (rank == 0) {
      // ---------------------------------------------- MMA issuer, padded mode
      unsigned long long af = 0, at = 0;
#define PCNN_PM_ISSUE(SL, MS) \
  mma_issuer_pm<ST, CG, SL, MS>(a, sbase, sA, sBp, pm_b_bytes, tmem_base, pair, npairs, pm_nj, &af, &at)
      if (a.msub == 2) {
        if (slab_bytes == 128) PCNN_PM_ISSUE(128, 2);
        else if (slab_bytes == 64) PCNN_PM_ISSUE(64, 2);
        else PCNN_PM_ISSUE(32, 2);
      } else {
        if (slab_bytes == 128) PCNN_PM_ISSUE(128, 1);
        else if (slab_bytes == 64) PCNN_PM_ISSUE(64, 1);
        else PCNN_PM_ISSUE(32, 1);
      }
#undef PCNN_PM_ISSUE
      if (TC_PROF(a) && lane == 0) {
        atomicAdd(&g_tc_prof[1], af);
        atomicAdd(&g_tc_prof[2], at);
      }
    }
  } else if (warp == 0) {
    // ------------------------------------------------ TMA producer (A im2col + B)
    if (lane == 0) {
      asm volatile("prefetch.tensormap [%0];" ::"l"((uint64_t)&tmap_w) : "memory");
      asm volatile("prefetch.tensormap [%0];" ::"l"((uint64_t)&tmap_x) : "memory");
      uint32_t stage = 0, phase = 0;
      WaitClock wc{TC_PROF(a) != 0};
      unsigned long long nkb = 0;
      for (int u = pair; u < a.units; u += npairs) {
        int mt, nt, grp, sp, k0, k1;
        decode(u, mt, nt, grp, sp);
        kb_range(sp, k0, k1);
        nkb += k1 - k0;
        const int nrow = grp * g.Nfg + nt * a.bn + (int)rank * b_rows;
        // input-space corner of this CTA's first output pixel (im2col) or of
        // its output rectangle (rect mode)
        int n0, w0, h0;
        if (rect) {
          const int ri = mt * CG + (int)rank;
          const int rw = ri % a.rects_w, rt = ri / a.rects_w;
          n0 = (rt / a.rects_h) * a.rect_n;
          h0 = (rt % a.rects_h) * a.rect_h - g.pad;
          w0 = rw * a.rect_w - g.pad;
        } else {
          const int m0 = mt * (TC_BM * CG) + (int)rank * TC_BM;
          n0 = m0 / HoWo;
          const int pq = m0 % HoWo;
          // perforated variant: kept positions psh / psw output rows / cols
          // apart; a zero-haloed input (shared-halo grid, interior at the
          // origin) only widens the map's extent
          w0 = (pq % g.Wo) * g.stride * max(g.psw, 1) - g.pad;
          h0 = (pq / g.Wo) * g.stride * max(g.psh, 1) - g.pad;
        }
        for (int kb = k0; kb < k1; ++kb) {
          wc.wait(sbase + SM_EMPTY + 8 * stage, phase ^ 1);
          const uint32_t fb = sbase + SM_FULL + 8 * stage;
          if (rank == 0)
            mbar_arrive_expect_tx(fb, CG * (((a.skip & 1) ? 0 : a_bytes) +
                                            ((a.skip & 2) ? 0 : b_stage)));
          const uint32_t dA = sA + stage * TC_A_STAGE;
          for (int sl = 0; sl < ((a.skip & 1) ? 0 : nslab); ++sl) {
            const int ke = kb * (TC_ROW_BYTES / ESZ) + sl * slab_elems;   // K element
            int r = 0, s = 0, c = ke;
            if (use_tab) {
              const uint32_t e = ktab_s[ke / slab_elems];
              r = (e >> 24) & 0xFF;
              s = (e >> 16) & 0xFF;
              c = e & 0xFFFF;
              if (r == 0xFF) { r = 0; s = 0; c = g.Cs; }   // beyond K: zero-fill
            } else if (ke >= g.K) {
              c = g.Cs;
            }
            const int cc = c >= g.Cs ? g.Cs : grp * g.Cg + c;
            const uint32_t dst = dA + sl * (TC_BM * slab_bytes);
            if (rect)
              tma_load_4d<CG>(dst, &tmap_x, fb, cc, w0 + s, h0 + r, n0);
            else if constexpr (CG == 1)
              tma_im2col(dst, &tmap_x, fb, cc, w0, h0, n0, (uint16_t)s, (uint16_t)r);
            else
              tma_im2col_2sm(dst, &tmap_x, fb, cc, w0, h0, n0, (uint16_t)s, (uint16_t)r);
          }
          if (!(a.skip & 2)) {
            if constexpr (CG == 1)
              tma_load_2d(sB + stage * b_stage, &tmap_w, fb, kb * (TC_ROW_BYTES / ESZ), nrow);
            else
              tma_load_2d_2sm(sB + stage * b_stage, &tmap_w, fb, kb * (TC_ROW_BYTES / ESZ), nrow);
          }
          advance(stage, phase, stages);
        }
      }
      if (TC_PROF(a)) {
        atomicAdd(&g_tc_prof[0], wc.acc);
        atomicAdd(&g_tc_prof[5], nkb);
      }
    }
  } else if (warp == 1) {
    if (rank == 0) {
      // ---------------------------------------------- MMA issuer (leader)
      unsigned long long af = 0, at = 0;
      if (slab_bytes == 128)
        mma_issuer_im2col<ST, CG, 128>(a, sbase, sA, sB, b_stage, tmem_base, pair, npairs, &af, &at);
      else if (slab_bytes == 64)
        mma_issuer_im2col<ST, CG, 64>(a, sbase, sA, sB, b_stage, tmem_base, pair, npairs, &af, &at);
      else
        mma_issuer_im2col<ST, CG, 32>(a, sbase, sA, sB, b_stage, tmem_base, pair, npairs, &af, &at);
      if (TC_PROF(a) && lane == 0) {
        atomicAdd(&g_tc_prof[1], af);
        atomicAdd(&g_tc_prof[2], at);
      }
    }
  } else {
    // ------------------------------------------------ epilogue (warps 2..)
    const int quarter = warp & 3;               // TMEM lanes 32*quarter..
    const int half = (warp - 2) >> 2;           // column half (8-warp epilogue)
    const int row = quarter * 32 + lane;
    const bool partial = a.splits > 1;
    uint8_t *stage = smem + SM_EPI + (warp - 2) * EPI_WARP_BYTES;
    const uint32_t tempty_leader =
        CG == 2 ? mapa(sbase + SM_TEMPTY, 0) : sbase + SM_TEMPTY;
    uint32_t lt = 0;
    uint32_t sbox = 0;   // bf16 TMA-store staging: two 2 KB boxes used alternately
    bool wide_prev = false;   // the last TMA store was a 64-column (4 KB) box
    unsigned long long ep_cmp = 0, ep_box = 0, ep_st = 0, ep_fence = 0, ep_issue = 0, ep_n = 0;   // profile (warp 2)
    // two warps per TMEM lane quarter: they split the N tile's columns at a
    // 32 boundary, or -- bf16 TMA stores of an N tile <= 64 with two M
    // sub-tiles -- take one sub-tile each with all its columns (64-column
    // boxes instead of two 32-column ones)
    const bool sub_split = a.tma_y && a.tma_y64 && a.msub == 2 && a.bn <= 64;
    const int csplit = sub_split ? a.bn : ((a.bn / 2 + 31) / 32) * 32;
    const int cbeg = sub_split || half == 0 ? 0 : csplit;
    const int cend = sub_split || half != 0 ? a.bn : csplit;
    WaitClock wtf{TC_PROF(a) != 0 && lane == 0 && warp == 2};
    unsigned long long busy = 0;
    long long tb = 0;
    for (int u = pair; u < a.units; u += npairs, ++lt) {
      int mt, nt, grp, sp;
      decode(u, mt, nt, grp, sp);
      const uint32_t buf = lt % a.nbuf, use = lt / a.nbuf;
      if (wtf.on && tb) busy += clock64() - tb;
      wtf.wait(sbase + SM_TFULL + 8 * buf, use & 1);
      if (wtf.on) tb = clock64();
      if (TC_PROF(a) && tl_first == 0) tl_first = gtimer();
      tc_fence_after();
      for (int sb = 0; sb < a.msub; ++sb) {
      if (sub_split && sb != half) continue;
      // TMEM columns of this sub-tile's accumulator
      const uint32_t tcol = buf * a.tbw + sb * a.tsub;
      int m;
      bool mok;
      if (rect) {
        const int ri = mt * CG + (int)rank;
        const int rw = ri % a.rects_w, rt = ri / a.rects_w;
        const int wi = row % a.rect_w, hr = row / a.rect_w;
        const int hi = hr % a.rect_h, ni = hr / a.rect_h;
        const int n = (rt / a.rects_h) * a.rect_n + ni;
        const int p = (rt % a.rects_h) * a.rect_h + hi, q = rw * a.rect_w + wi;
        mok = row < rect_rows && q < g.Wo && p < g.Ho && n * HoWo < g.M;
        m = (n * g.Ho + p) * g.Wo + q;
      } else {
        m = ((mt * CG + (int)rank) * a.msub + sb) * TC_BM + row;
        mok = m < g.M;
      }
      bool valid = true;      // padded mode: halo rows are stored as zeros
      if (g.pm == 2) {
        // row-perforated: MMA row = (kept row k of the tile, grid column v;
        // segments are wv + 2 pad long).  m = the kept row's own position on
        // the layer's output grid; the store below copies it to every output
        // row whose nearest kept row it is (R13), halo columns as zeros.
        const int T = (mt * CG + (int)rank) * a.msub + sb, n = T / g.tpi, tb = T - n * g.tpi;
        const int k = (int)a.fd_w.div((uint32_t)row), v = row - k * (g.wv + 2 * g.pad);
        const int pk = tb * g.nseg + k;
        mok = k < g.nseg && pk < g.hk && v < g.wv && T * TC_BM < g.M;
        m = (n * g.hv + g.vh + pk * g.psh) * g.wv + v;
        valid = mok && v >= g.vh && v < g.vh + g.Wo;
      } else if (g.pm) {
        const int ni = (int)a.fd_hw.div((uint32_t)m), rem = m - ni * g.hv * g.wv;
        const int pv = (int)a.fd_w.div((uint32_t)rem), qv = rem - pv * g.wv;
        valid = pv >= g.vh && pv < g.vh + g.Ho && qv >= g.vh && qv < g.vh + g.Wo;
      }
      const size_t orow = (size_t)m * g.out_cs;
      if constexpr (LRN) {
        epilogue_lrn<ST>(a, tmem_base + ((uint32_t)(quarter * 32) << 16) + tcol, mok,
                         valid, orow, stage, lane, half);
        continue;
      }
      if (a.tma_y) {
        // Full chunks are staged in this warp's swizzled box and leave by one
        // TMA tensor store of the warp's 32 rows (rows past M are clipped by
        // the map); a ragged last chunk falls back to row stores.  BF16
        // chunks are 64 columns (128 B rows, SW128, 4 KB box) where the range
        // allows, else 32 columns (SW64, 2 KB boxes used alternately, so a
        // chunk waits only for the store issued two chunks earlier).  The
        // TMA store cost grows with the box-row count, so narrow-N layers
        // (AlexNet conv1, VGG conv1_x, the rank-r second stage) move 128 B
        // per row request instead of 64 B.  FP32 chunks are 32 columns
        // (128 B rows, SW128).
        const bool o16 = g.out_mode == OUT_BF16;
        const int row0 = m - lane;                       // the warp's first row
        const uint32_t trow = tmem_base + ((uint32_t)(quarter * 32) << 16) + tcol;
        for (int c0 = cbeg; c0 < cend;) {
          const int n = nt * a.bn + c0;
          if (n >= g.Nfg) break;                         // warp-uniform
          const int col = grp * g.Nfg + n;
          const bool w64 = a.tma_y64 && c0 + 64 <= cend && n + 64 <= g.Nfg;
          const bool full = w64 || (n + 32 <= g.Nfg && c0 + 32 <= cend);
          if (!full) {
            // ragged chunk: row stores of the np valid 16 B pieces
            float f[32];
            epi_chunk32(a, trow + c0, col, valid, f);
            uint4 pc[8];
            const int eb = o16 ? 2 : 4;
            if (o16) {
#pragma unroll
              for (int q = 0; q < 4; ++q) pc[q] = pack_bf16x8(f + 8 * q);
            } else {
              const bool rnd = g.out_mode == OUT_F32_TF32;
#pragma unroll
              for (int q = 0; q < 8; ++q) {
                float t[4];
#pragma unroll
                for (int i = 0; i < 4; ++i) t[i] = rnd ? tf32_rna_tc(f[4 * q + i]) : f[4 * q + i];
                pc[q] = make_uint4(__float_as_uint(t[0]), __float_as_uint(t[1]),
                                   __float_as_uint(t[2]), __float_as_uint(t[3]));
              }
            }
            if (lane == 0) bulk_wait_read0();
            __syncwarp();
            const int np = min(o16 ? 4 : 8, (min(g.Nfg - n, cend - c0) * eb) / 16);
            char *rowp = mok ? (char *)a.y + ((size_t)m * g.out_cs + col) * eb : nullptr;
            epi_store_rows(stage, pc, np, rowp, lane);
            c0 += 32;
            continue;
          }
          // first 32 columns computed while earlier stores drain, then the
          // staging box must be free: a 64-column box (or any chunk after
          // one) needs every earlier store to have read its source
          const bool pon = TC_PROF(a) && warp == 2;
          long long pt = pon ? clock64() : 0;
          float f[32];
          epi_chunk32(a, trow + c0, col, valid, f);
          if (pon) { const long long t = clock64(); ep_cmp += t - pt; pt = t; }
          if (lane == 0) {
            if (o16 && !w64 && !wide_prev) bulk_wait_read1();
            else bulk_wait_read0();
          }
          __syncwarp();
          if (pon) { const long long t = clock64(); ep_box += t - pt; pt = t; }
          if (w64) {
#pragma unroll
            for (int q = 0; q < 4; ++q)
              *(uint4 *)(stage + lane * 128 + ((q ^ (lane & 7)) << 4)) = pack_bf16x8(f + 8 * q);
            if (pon) { const long long t = clock64(); ep_st += t - pt; pt = t; }
            epi_chunk32(a, trow + c0 + 32, col + 32, valid, f);
            if (pon) { const long long t = clock64(); ep_cmp += t - pt; pt = t; }
#pragma unroll
            for (int q = 0; q < 4; ++q)
              *(uint4 *)(stage + lane * 128 + (((4 + q) ^ (lane & 7)) << 4)) = pack_bf16x8(f + 8 * q);
          } else if (o16) {
            uint8_t *box = stage + sbox * 2048;
#pragma unroll
            for (int q = 0; q < 4; ++q)
              *(uint4 *)(box + lane * 64 + ((q ^ ((lane >> 1) & 3)) << 4)) = pack_bf16x8(f + 8 * q);
          } else {
            const bool rnd = g.out_mode == OUT_F32_TF32;
#pragma unroll
            for (int q = 0; q < 8; ++q) {
              float t[4];
#pragma unroll
              for (int i = 0; i < 4; ++i) t[i] = rnd ? tf32_rna_tc(f[4 * q + i]) : f[4 * q + i];
              *(uint4 *)(stage + lane * 128 + ((q ^ (lane & 7)) << 4)) =
                  make_uint4(__float_as_uint(t[0]), __float_as_uint(t[1]),
                             __float_as_uint(t[2]), __float_as_uint(t[3]));
            }
          }
          if (pon) { const long long t = clock64(); ep_st += t - pt; pt = t; }
          fence_proxy_async();
          __syncwarp();
          if (pon) { const long long t = clock64(); ep_fence += t - pt; pt = t; }
          if (lane == 0 && row0 < g.M) {
            if (w64) tma_store_2d(&tmap_y64, smem_u32(stage), col, row0);
            else tma_store_2d(&tmap_y, smem_u32(o16 ? stage + sbox * 2048 : stage), col, row0);
            bulk_commit();
          }
          if (pon) { ep_issue += clock64() - pt; ++ep_n; }
          if (o16 && !w64) sbox ^= 1;
          wide_prev = w64;
          c0 += w64 ? 64 : 32;
        }
        continue;
      }
      // bias is zero-padded on the device, so whole float4s can be read.
      // Each pass drains 128 B of every row: 64 bf16 or 32 fp32 columns.
      const bool out16 = !partial && g.out_mode == OUT_BF16;
      const int pass_cols = out16 ? 64 : 32;
      const int ocs = partial ? g.out_cs : g.out_cs;
      char *obase = partial ? (char *)(a.ws + (size_t)sp * g.M * g.out_cs)
                            : (char *)a.y;
      const int eb = out16 ? 2 : 4;
      for (int c0 = cbeg; c0 < cend; c0 += pass_cols) {
        const int n = nt * a.bn + c0;          // column within the group
        if (n >= g.Nfg) break;                 // warp-uniform
        const int col = grp * g.Nfg + n;
        float f[64];
#pragma unroll
        for (int h = 0; h < 2; ++h) {
          if (h == 0 || (out16 && c0 + 32 < cend)) {
            uint32_t v[32];
            tmem_ld32(tmem_base + ((uint32_t)(quarter * 32) << 16) + tcol + c0 + 32 * h, v);
            tmem_ld_wait();
#pragma unroll
            for (int i = 0; i < 32; ++i) f[32 * h + i] = __uint_as_float(v[i]);
          }
        }
        if (!partial) {
          const float4 *bp = (const float4 *)(a.bias + col);
#pragma unroll
          for (int q = 0; q < 16; ++q) {
            if (q < 8 || out16) {
              const float4 bb = __ldg(bp + q);
              f[4 * q] += bb.x;
              f[4 * q + 1] += bb.y;
              f[4 * q + 2] += bb.z;
              f[4 * q + 3] += bb.w;
            }
          }
          if (g.relu)
#pragma unroll
            for (int i = 0; i < 64; ++i) f[i] = fmaxf(f[i], 0.f);
          if (!valid)
#pragma unroll
            for (int i = 0; i < 64; ++i) f[i] = 0.f;
        }
        uint4 pc[8];
        if (out16) {
#pragma unroll
          for (int q = 0; q < 8; ++q) {
            uint32_t *pw = (uint32_t *)&pc[q];
#pragma unroll
            for (int i = 0; i < 4; ++i) {
              __nv_bfloat162 b2 = __floats2bfloat162_rn(f[8 * q + 2 * i], f[8 * q + 2 * i + 1]);
              pw[i] = *(uint32_t *)&b2;
            }
          }
        } else {
          const bool rnd = !partial && g.out_mode == OUT_F32_TF32;
#pragma unroll
          for (int q = 0; q < 8; ++q) {
            float t[4];
#pragma unroll
            for (int i = 0; i < 4; ++i) t[i] = rnd ? tf32_rna_tc(f[4 * q + i]) : f[4 * q + i];
            pc[q] = make_uint4(__float_as_uint(t[0]), __float_as_uint(t[1]),
                               __float_as_uint(t[2]), __float_as_uint(t[3]));
          }
        }
        // pieces of this pass inside both the group (Nfg) and this N tile (bn)
        const int np = min(8, (min(min(g.Nfg - n, cend - c0), pass_cols) * eb) / 16);
        char *rowp = mok ? obase + ((size_t)m * ocs + col) * eb : nullptr;
        if (g.pm == 2) {
          // kept output row p = pk * psh -> every row q with nearest kept row p
          const int p = m / g.wv % g.hv - g.vh;
          for (int d = -((g.psh - 1) / 2); d < g.psh; ++d) {     // warp-uniform bounds
            const int q = p + d;
            bool ok = rowp != nullptr && q >= 0 && q < g.Ho;
            if (ok) {
              const int lo = q / g.psh * g.psh, hi = lo + g.psh;
              ok = ((hi < g.Ho && hi - q < q - lo) ? hi : lo) == p;
            }
            epi_store_rows(stage, pc, np,
                           ok ? rowp + (ptrdiff_t)d * g.wv * ocs * eb : nullptr, lane);
          }
        } else {
          epi_store_rows(stage, pc, np, rowp, lane);
        }
      }
      }   // sub-tiles
      tc_fence_before();
      __syncwarp();
      if (lane == 0) {
        if (CG == 2 && rank != 0) mbar_arrive_cluster(tempty_leader + 8 * buf);
        else mbar_arrive(sbase + SM_TEMPTY + 8 * buf);
      }
    }
    if (lane == 0) bulk_wait0();                 // TMA stores complete before exit
    __syncwarp();
    if (wtf.on && tb) busy += clock64() - tb;
    wtf_acc_out = wtf.acc;
    busy_out = busy;
    if (TC_PROF(a) && warp == 2 && lane == 0) {
      atomicAdd(&g_tc_prof[17], tl_first - tl_wait);
      atomicAdd(&g_tc_prof[18], gtimer() - tl_wait);
      atomicAdd(&g_tc_prof[8], ep_cmp);
      atomicAdd(&g_tc_prof[9], ep_box);
      atomicAdd(&g_tc_prof[10], ep_st);
      atomicAdd(&g_tc_prof[11], ep_n);
      atomicAdd(&g_tc_prof[12], ep_fence);
      atomicAdd(&g_tc_prof[13], ep_issue);
    }
  }

  if (TC_PROF(a) && warp == 2 && lane == 0) {
    atomicAdd(&g_tc_prof[3], wtf_acc_out);
    atomicAdd(&g_tc_prof[6], busy_out);
  }
  tc_fence_before();
  if constexpr (CG == 2) cluster_sync(); else __syncthreads();
  tc_fence_after();
  if (TC_PROF(a) && tid == 0) {
    atomicAdd(&g_tc_prof[4], (unsigned long long)(clock64() - t_start));
    atomicAdd(&g_tc_prof[7], 1ULL);
    const unsigned long long tl_exit = gtimer();
    atomicAdd(&g_tc_prof[16], tl_wait - tl_entry);
    atomicAdd(&g_tc_prof[19], tl_exit - tl_wait);
    atomicAdd(&g_tc_prof[20], 1ULL);
    atomicMax(&g_tc_prof[21], ~tl_entry);
    atomicMax(&g_tc_prof[22], tl_exit);
    atomicMax(&g_tc_prof[23], ~tl_wait);
    atomicMax(&g_tc_prof[24], tl_wait);
  }
  if (warp == 1) {
    if constexpr (CG == 1)
      asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem_base),
                   "n"(TC_TMEM_COLS));
    else
      asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, %1;" ::"r"(tmem_base),
                   "n"(TC_TMEM_COLS));
  }
}

// Deterministic split-K reduction: y = act(sum_s ws[s] + bias), s ascending.
// Padded-layout (pm) GEMMs: rows outside the valid window of the grid are
// stored as zeros (pm_hv > 0: grid hv x wv per image, valid [vh, vh + Ho) x
// [vh, vh + Wo)).
__global__ void splitk_reduce_kernel(const float *__restrict__ ws, void *y,
                                     const float *__restrict__ bias, int M, int N, int splits,
                                     int relu, int out_mode, int pm_hv, int pm_wv, int pm_vh,
                                     int pm_ho, int pm_wo) {
  pdl_enter();
  const long long total = (long long)M * N / 4;
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < total;
       i += (long long)gridDim.x * blockDim.x) {
    const long long e = i * 4;
    const int col = (int)(e % N);
    if (pm_hv > 0) {
      const long long m = e / N;
      const int rem = (int)(m % ((long long)pm_hv * pm_wv));
      const int pv = rem / pm_wv, qv = rem - pv * pm_wv;
      if (pv < pm_vh || pv >= pm_vh + pm_ho || qv < pm_vh || qv >= pm_vh + pm_wo) {
        if (out_mode == OUT_BF16) *(uint2 *)((__nv_bfloat16 *)y + e) = make_uint2(0, 0);
        else *(float4 *)((float *)y + e) = make_float4(0.f, 0.f, 0.f, 0.f);
        continue;
      }
    }
    // partials summed in split order (fixed, so every SM budget gives the
    // same bits); the loads of three splits are issued before their adds so
    // a thread has three L2 round trips in flight instead of one
    const size_t sMN = (size_t)M * N;
    float4 acc = *(const float4 *)(ws + e);
    int s = 1;
    for (; s + 2 < splits; s += 3) {
      const float4 v0 = *(const float4 *)(ws + (size_t)s * sMN + e);
      const float4 v1 = *(const float4 *)(ws + (size_t)(s + 1) * sMN + e);
      const float4 v2 = *(const float4 *)(ws + (size_t)(s + 2) * sMN + e);
      acc.x = ((acc.x + v0.x) + v1.x) + v2.x;
      acc.y = ((acc.y + v0.y) + v1.y) + v2.y;
      acc.z = ((acc.z + v0.z) + v1.z) + v2.z;
      acc.w = ((acc.w + v0.w) + v1.w) + v2.w;
    }
    for (; s < splits; ++s) {
      const float4 v = *(const float4 *)(ws + (size_t)s * sMN + e);
      acc.x += v.x;
      acc.y += v.y;
      acc.z += v.z;
      acc.w += v.w;
    }
    float f[4] = {acc.x, acc.y, acc.z, acc.w};
#pragma unroll
    for (int t = 0; t < 4; ++t) {
      if (bias) f[t] += __ldg(&bias[col + t]);
      if (relu) f[t] = fmaxf(f[t], 0.f);
    }
    if (out_mode == OUT_BF16) {
      __nv_bfloat162 lo = __floats2bfloat162_rn(f[0], f[1]);
      __nv_bfloat162 hi = __floats2bfloat162_rn(f[2], f[3]);
      uint2 pk = make_uint2(*(uint32_t *)&lo, *(uint32_t *)&hi);
      *(uint2 *)((__nv_bfloat16 *)y + e) = pk;
    } else {
      if (out_mode == OUT_F32_TF32)
        for (int t = 0; t < 4; ++t) f[t] = tf32_rna_tc(f[t]);
      *(float4 *)((float *)y + e) = make_float4(f[0], f[1], f[2], f[3]);
    }
  }
}

template <int ST, int CG, bool LRN>
static cudaError_t set_smem_attr() {
  return cudaFuncSetAttribute(conv_tc_kernel<ST, CG, LRN>,
                              cudaFuncAttributeMaxDynamicSharedMemorySize, (int)TC_SMEM_BYTES);
}

cudaError_t tc_init() {
  cudaError_t e;
  if ((e = set_smem_attr<ST_BF16, 1, false>()) != cudaSuccess) return e;
  if ((e = set_smem_attr<ST_BF16, 2, false>()) != cudaSuccess) return e;
  if ((e = set_smem_attr<ST_F32, 1, false>()) != cudaSuccess) return e;
  if ((e = set_smem_attr<ST_F32, 2, false>()) != cudaSuccess) return e;
  if ((e = set_smem_attr<ST_BF16, 1, true>()) != cudaSuccess) return e;
  if ((e = set_smem_attr<ST_BF16, 2, true>()) != cudaSuccess) return e;
  if ((e = set_smem_attr<ST_F32, 1, true>()) != cudaSuccess) return e;
  return set_smem_attr<ST_F32, 2, true>();
}

int tc_slab_bytes(int st, int cg_channels) {
  const int esz = st == ST_BF16 ? 2 : 4;
  for (int sb = 128; sb >= 32; sb >>= 1)
    if ((cg_channels * esz) % sb == 0) return sb;
  return 0;   // channels per group must be a multiple of 32 bytes
}

template <int ST, int CG, bool LRN>
static cudaError_t launch_tc(const CUtensorMap *tmap_w, const CUtensorMap *tmap_x,
                             const CUtensorMap *tmap_y, const CUtensorMap *tmap_y64,
                             const TcArgs &args, int grid, cudaStream_t s) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(grid);
  cfg.blockDim = dim3(tc_threads<LRN>());
  cfg.dynamicSmemBytes = TC_SMEM_BYTES;
  cfg.stream = s;
  cudaLaunchAttribute attr[2];
  attr[0].id = cudaLaunchAttributeClusterDimension;
  attr[0].val.clusterDim.x = CG;
  attr[0].val.clusterDim.y = 1;
  attr[0].val.clusterDim.z = 1;
  attr[1].id = cudaLaunchAttributeProgrammaticStreamSerialization;   // PDL
  attr[1].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 2;
  return cudaLaunchKernelEx(&cfg, conv_tc_kernel<ST, CG, LRN>, *tmap_w, *tmap_x, *tmap_y, *tmap_y64,
                            args);
}

cudaError_t tc_profile(int reset, unsigned long long out[32]) {
  cudaError_t e = cudaDeviceSynchronize();
  if (e != cudaSuccess) return e;
  if (out) e = cudaMemcpyFromSymbol(out, g_tc_prof, sizeof(unsigned long long) * 32);
  if (e != cudaSuccess) return e;
  if (reset) {
    unsigned long long z[32] = {};
    e = cudaMemcpyToSymbol(g_tc_prof, z, sizeof(z));
  }
  return e;
}

cudaError_t launch_conv_tc(const ConvGeom &g, int st, const CUtensorMap *tmap_x,
                           const CUtensorMap *tmap_w, const float *bias, void *y,
                           const int *ktab, const TcPlan &p, float *ws, const Budget &b,
                           cudaStream_t s, const float *lrn, const CUtensorMap *tmap_y,
                           const CUtensorMap *tmap_y64) {
  TcArgs args;
  static const int prof_env = [] {
    const char *e = exp_env("PCNN_TC_PROFILE");
    return e && e[0] == '1' ? 1 : 0;
  }();
  static const int skip_env = [] {
    const char *e = exp_env("PCNN_TC_SKIP");
    return e ? atoi(e) : 0;
  }();
  args.prof = prof_env;
  args.skip = skip_env;
  args.lrn = 0;
  args.lrn_a_over_n = args.lrn_beta = args.lrn_k = 0.f;
  if (lrn) {   // {size, alpha, beta, k}: size 5 only, one N tile with every channel
    if (lrn[0] != 5.f || p.ntiles != 1 || g.groups != 1 || p.splits != 1 || g.Nfg > 128 ||
        p.bn != ((g.Nfg + 31) / 32) * 32)
      return cudaErrorInvalidValue;
    args.lrn = 1;
    args.lrn_a_over_n = lrn[1] / lrn[0];
    args.lrn_beta = lrn[2];
    args.lrn_k = lrn[3];
  }
  args.g = g;
  args.fd_mt.init(p.mtiles);
  args.fd_nt.init(p.ntiles);
  args.fd_grp.init(g.groups);
  args.fd_hw.init(g.pm ? g.hv * g.wv : 1);
  args.fd_w.init(g.pm == 2 ? g.wv + 2 * g.pad : g.pm ? g.wv : 1);
  args.y = y;
  args.tma_y = (tmap_y != nullptr && !lrn && p.splits == 1 && p.rect_w == 0 && g.pm != 2) ? 1 : 0;
  args.tma_y64 = args.tma_y && tmap_y64 != nullptr && g.out_mode == OUT_BF16 ? 1 : 0;
  const CUtensorMap *ym = tmap_y ? tmap_y : tmap_x;
  const CUtensorMap *ym64 = args.tma_y64 ? tmap_y64 : ym;
  args.ws = ws;
  args.bias = bias;
  args.ktab = ktab;
  args.bn = p.bn;
  args.mtiles = p.mtiles;
  args.ntiles = p.ntiles;
  args.splits = p.splits;
  args.units = p.units;
  args.kblocks = g.Kpad / tc_block_k_elems(st);
  args.kb_per_split = p.kb_per_split;
  args.stages = tc_stages_for(p.bn, p.cg);
  args.slab_bytes = tc_slab_bytes(st, g.Cg);
  args.rect_w = p.rect_w;
  args.rect_h = p.rect_h;
  args.rect_n = p.rect_n;
  args.rects_w = p.rect_w ? (g.Wo + p.rect_w - 1) / p.rect_w : 0;
  args.rects_h = p.rect_w ? (g.Ho + p.rect_h - 1) / p.rect_h : 0;
  args.a_stages = p.a_stages;
  args.b_stages = p.b_stages;
  args.msub = p.msub > 1 ? p.msub : 1;
  {
    // TMEM ring: sub-tile stride = the N tile rounded to 32 columns, buffer
    // width = msub strides rounded up to a power of two (>= 64), as many
    // buffers as fit the 512 allocated columns (2 .. 8)
    args.tsub = (p.bn + 31) / 32 * 32;
    int w = 64;
    while (w < args.msub * args.tsub) w <<= 1;
    args.tbw = w;
    args.nbuf = std::min(TC_MAX_TBUF, TC_TMEM_COLS / w);
    if (const char *e = exp_env("PCNN_TC_NBUF")) args.nbuf = std::max(2, std::min(args.nbuf, atoi(e)));
  }
  {
    // padded mode: UMMAs of the last channel slab that reach real channels
    const int se = args.slab_bytes / (st == ST_BF16 ? 2 : 4);
    const int creal = g.Creal > 0 && g.Creal <= g.Cg ? g.Creal : g.Cg;
    const int ncb = se > 0 ? g.Cg / se : 1;
    const int valid_b = (creal - (ncb - 1) * se) * (st == ST_BF16 ? 2 : 4);
    const char *ek = exp_env("PCNN_NO_KSKIP");           // A/B: multiply the padding too
    args.kmma_last = args.slab_bytes / 32;
    if (!(ek && ek[0] == '1') && valid_b > 0)
      args.kmma_last = std::min(args.slab_bytes / 32, (valid_b + 31) / 32);
  }
  args.ww = g.pm == 1 ? p.ww : 0;
  args.pm_rows = g.pm ? pm_window_rows(g.S, g.wv, args.ww) : 0;
  args.pm_sub = (args.pm_rows + 7) / 8 * 8;
  args.pm_a_stage = g.pm ? pm_a_stage_bytes(args.slab_bytes, args.pm_rows, args.msub) : 0;
  if (args.ww && (p.splits != 1 || args.pm_rows > 256)) return cudaErrorInvalidValue;
  if (args.msub > 2 || (args.msub == 2 && (!g.pm || p.bn > TC_BN_MAX / 2)) ||
      (g.pm == 2 && (g.nseg < 1 || g.nseg * (g.wv + 2 * g.pad) > TC_BM || g.tpi < 1)))
    return cudaErrorInvalidValue;
  args.b = b;
  if (args.slab_bytes == 0) return cudaErrorInvalidValue;
  if (g.pm && ((p.splits != 1 && g.pm != 1) || p.rect_w || g.stride != 1 ||
               (g.S != 2 * g.pad + 1 && g.pad != 0) ||
               g.Cg % (args.slab_bytes / (st == ST_BF16 ? 2 : 4)) || p.a_stages < 2 ||
               p.b_stages < 2 || p.a_stages > TC_MAX_ASTAGES || p.b_stages > TC_MAX_BSTAGES))
    return cudaErrorInvalidValue;
  cudaError_t e;
  const bool L = args.lrn != 0;
  if (st == ST_BF16)
    e = p.cg == 2 ? (L ? launch_tc<ST_BF16, 2, true>(tmap_w, tmap_x, ym, ym64, args, p.grid, s)
                       : launch_tc<ST_BF16, 2, false>(tmap_w, tmap_x, ym, ym64, args, p.grid, s))
                  : (L ? launch_tc<ST_BF16, 1, true>(tmap_w, tmap_x, ym, ym64, args, p.grid, s)
                       : launch_tc<ST_BF16, 1, false>(tmap_w, tmap_x, ym, ym64, args, p.grid, s));
  else
    e = p.cg == 2 ? (L ? launch_tc<ST_F32, 2, true>(tmap_w, tmap_x, ym, ym64, args, p.grid, s)
                       : launch_tc<ST_F32, 2, false>(tmap_w, tmap_x, ym, ym64, args, p.grid, s))
                  : (L ? launch_tc<ST_F32, 1, true>(tmap_w, tmap_x, ym, ym64, args, p.grid, s)
                       : launch_tc<ST_F32, 1, false>(tmap_w, tmap_x, ym, ym64, args, p.grid, s));
  if (e != cudaSuccess) return e;
  e = cudaGetLastError();
  if (e != cudaSuccess || p.splits <= 1) return e;
  const long long total = (long long)g.M * g.out_cs / 4;
  const int grid = (int)std::min<long long>((total + 255) / 256, 148 * 8);
  launch_pdl(splitk_reduce_kernel, dim3(grid), dim3(256), 0, s, ws, y, bias, g.M, g.out_cs, p.splits, g.relu,
             g.out_mode, g.pm == 1 ? g.hv : 0, g.wv, g.vh, g.Ho, g.Wo);
  return cudaGetLastError();
}

}  // namespace pcnn
