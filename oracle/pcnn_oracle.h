/*
 * pcnn_oracle.h -- FP64 CPU oracle for the P-CNN inference hot path.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and
 * bench.py's cpu_baseline / --impl reference legs may load this library.
 * It shares no code, header, table or helper with the CUDA path
 * (paper_conf_hpca_songhcl17_b200/ and include/pcnn.h).
 *
 * Every function is a plain, slow, obviously-correct loop in double
 * precision following the passage of PAPER.md (cited as P:<line>) that
 * defines it.  Layouts are the paper's / Caffe's: activations NCHW,
 * conv weights OIHW (F_m of Fig. 2 row-major = [N_f][N_c/g][S_f][S_f]),
 * FC weights [out][in] with the input flattened in C,H,W order.
 *
 * Threading: functions taking `nthreads` split independent work items
 * (an image, or one output channel / feature of one image) over pthreads;
 * every output value is computed by one sequential loop, so the result does
 * not depend on nthreads.
 *
 * Return value: 0 on success, negative on bad arguments.
 */
#ifndef PCNN_ORACLE_H
#define PCNN_ORACLE_H

#ifdef __cplusplus
extern "C" {
#endif

/* Output size of a convolution: floor((H + 2 pad - S) / stride) + 1. */
int orc_conv_out_size(int in, int k, int stride, int pad);
/* Output size of a pooling layer, Caffe ceil mode (no padding). */
int orc_pool_out_size(int in, int k, int stride);

/* P:55-59 (Fig. 2, eq. 1): y[n,f,p,q] = b_f + sum_{c,r,s} W[f,c,r,s] *
 * x[n, g(f)*C/g + c, p*st + r - pad, q*st + s - pad], zero outside the image;
 * optional ReLU (reading R2).  y is [B, F, Ho, Wo]. */
int orc_conv2d(const double *x, int B, int C, int H, int W,
               const double *w, const double *bias, int F, int S, int stride,
               int pad, int groups, int relu, double *y, int nthreads);

/* The same layer computed literally as Fig. 2 does it: im2col builds
 * D_m (S_f^2 N_c x W_o H_o, rows in (c, r, s) order) per group, then
 * O_m = F_m x D_m (+bias, ReLU).  Used to cross-check orc_conv2d. */
int orc_conv2d_im2col_gemm(const double *x, int B, int C, int H, int W,
                           const double *w, const double *bias, int F, int S,
                           int stride, int pad, int groups, int relu,
                           double *y);

/* Caffe across-channel LRN (reading R3):
 * y_c = x_c / (k + alpha/size * sum_{c' in window(c)} x_{c'}^2)^beta. */
int orc_lrn(const double *x, int B, int C, int H, int W, int size,
            double alpha, double beta, double k, double *y, int nthreads);

/* Max / average pooling, k x k window, stride s, no padding. */
int orc_maxpool(const double *x, int B, int C, int H, int W, int k,
                int stride, double *y, int nthreads);
int orc_avgpool(const double *x, int B, int C, int H, int W, int k,
                int stride, double *y, int nthreads);

/* Classifier (FC) layer: y[n,j] = b_j + sum_i W[j,i] x[n,i] (+ReLU). */
int orc_fc(const double *x, int B, int K, const double *w,
           const double *bias, int N, int relu, double *y, int nthreads);

/* P:89 + eq. 2: p = softmax(z), H = -sum p ln p (0 ln 0 = 0). */
int orc_softmax_entropy(const double *z, int B, int N, double *p, double *H);

/* Entropy of a given probability vector, eq. 2 (natural log). */
double orc_entropy(const double *p, int n);

/* Rank-r operator (reading R7): for one weight matrix
 * Wm (N x K, row-major), W_r = U_r U_r^T Wm where U_r holds the top-r
 * eigenvectors of the Gram matrix Wm Wm^T (cyclic Jacobi, FP64).
 * sigma (length min(N,K), may be NULL) receives the singular values
 * sqrt(max(eig,0)) in descending order.  Returns 0, or 1 if the r-th
 * singular value gap (sigma_r - sigma_{r+1}) / sigma_1 < 1e-6 (W_r not
 * unique), negative on error. */
int orc_rank_r(const double *Wm, int N, int K, int r, double *Wr,
               double *sigma);

/* Analytical helpers of P:186-211, P:281-303 (eqs. 4, 5, 6, 8, 9, 11). */
long orc_grid_size(long M, long N, long m, long n);                 /* eq. 4 */
long orc_max_blocks(long nSMs, long R, long block_size, long r);    /* eq. 5 */
double orc_util(long grid, long max_blocks);                        /* eq. 6 */
long orc_n_invocations(long grid, long tlp, long nSMs);             /* eq. 8 */
double orc_rec(long M, long N, long m, long n);                     /* eq. 9 */
long orc_opt_sm(long grid, long opt_tlp, long num_sms);             /* eq. 11 */

#ifdef __cplusplus
}
#endif
#endif
