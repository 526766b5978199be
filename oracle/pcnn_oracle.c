/*
 * pcnn_oracle.c -- FP64 CPU oracle for the P-CNN inference hot path.
 *
 * TEST INFRASTRUCTURE ONLY (see pcnn_oracle.h).  Plain loops, double
 * precision, no blocking, fusion or reordering beyond the definitions cited.
 * Parity pins for every function live in tests/test_oracle_*.py; none is
 * "parity unpinned".
 */
#include "pcnn_oracle.h"

#include <math.h>
#include <pthread.h>
#include <stdlib.h>
#include <string.h>

/* ------------------------------------------------------------------ */
/* work-item parallelism: every output value is computed sequentially  */
/* ------------------------------------------------------------------ */
typedef void (*image_fn)(void *ctx, int n);

typedef struct {
    image_fn fn;
    void *ctx;
    int B;
    int next;
    pthread_mutex_t mu;
} pool_t;

static void *pool_worker(void *arg) {
    pool_t *p = (pool_t *)arg;
    for (;;) {
        pthread_mutex_lock(&p->mu);
        int n = p->next++;
        pthread_mutex_unlock(&p->mu);
        if (n >= p->B) break;
        p->fn(p->ctx, n);
    }
    return NULL;
}

static void for_each_image(image_fn fn, void *ctx, int B, int nthreads) {
    if (nthreads <= 1 || B <= 1) {
        for (int n = 0; n < B; ++n) fn(ctx, n);
        return;
    }
    if (nthreads > B) nthreads = B;
    pool_t p;
    p.fn = fn; p.ctx = ctx; p.B = B; p.next = 0;
    pthread_mutex_init(&p.mu, NULL);
    pthread_t *th = (pthread_t *)malloc(sizeof(pthread_t) * (size_t)nthreads);
    int started = 0;
    for (int t = 0; t < nthreads; ++t)
        if (pthread_create(&th[t], NULL, pool_worker, &p) == 0) ++started;
    if (started == 0) pool_worker(&p);
    for (int t = 0; t < started; ++t) pthread_join(th[t], NULL);
    free(th);
    pthread_mutex_destroy(&p.mu);
}

/* ------------------------------------------------------------------ */
/* output sizes                                                        */
/* ------------------------------------------------------------------ */
int orc_conv_out_size(int in, int k, int stride, int pad) {
    /* reading R1(iii): floor((H + 2 pad - S)/stride) + 1 */
    if (stride <= 0 || in + 2 * pad < k) return -1;
    return (in + 2 * pad - k) / stride + 1;
}

int orc_pool_out_size(int in, int k, int stride) {
    /* reading R4: Caffe ceil mode, ceil((H - k)/s) + 1, no padding; the
     * last window must start inside the image. */
    if (stride <= 0 || in < k) return -1;
    int o = (in - k + stride - 1) / stride + 1;
    if ((o - 1) * stride >= in) --o;
    return o;
}

/* ------------------------------------------------------------------ */
/* convolution: direct definition (eq. 1, Fig. 2)              */
/* ------------------------------------------------------------------ */
typedef struct {
    const double *x, *w, *bias;
    double *y;
    int C, H, W, F, S, stride, pad, groups, relu, Ho, Wo;
} conv_ctx;

/* one work item = one output channel f of one image n */
static void conv_item(void *vctx, int item) {
    const conv_ctx *c = (const conv_ctx *)vctx;
    const int n = item / c->F, f = item % c->F;
    const int Cg = c->C / c->groups, Fg = c->F / c->groups;
    const int g = f / Fg;                           /* g(f) = floor(f / (N_f/g)) */
    for (int p = 0; p < c->Ho; ++p) {
        for (int q = 0; q < c->Wo; ++q) {
            double acc = 0.0;
            for (int ci = 0; ci < Cg; ++ci) {
                const int cin = g * Cg + ci;
                for (int r = 0; r < c->S; ++r) {
                    const int ih = p * c->stride + r - c->pad;
                    if (ih < 0 || ih >= c->H) continue;      /* zero padding */
                    for (int s = 0; s < c->S; ++s) {
                        const int iw = q * c->stride + s - c->pad;
                        if (iw < 0 || iw >= c->W) continue;
                        acc += c->w[(((size_t)f * Cg + ci) * c->S + r) * c->S + s] *
                               c->x[(((size_t)n * c->C + cin) * c->H + ih) * c->W + iw];
                    }
                }
            }
            double v = acc + (c->bias ? c->bias[f] : 0.0);
            if (c->relu && v < 0.0) v = 0.0;         /* reading R2 */
            c->y[(((size_t)n * c->F + f) * c->Ho + p) * c->Wo + q] = v;
        }
    }
}

int orc_conv2d(const double *x, int B, int C, int H, int W, const double *w,
               const double *bias, int F, int S, int stride, int pad,
               int groups, int relu, double *y, int nthreads) {
    if (!x || !w || !y || B < 0 || groups <= 0 || C % groups || F % groups)
        return -1;
    int Ho = orc_conv_out_size(H, S, stride, pad);
    int Wo = orc_conv_out_size(W, S, stride, pad);
    if (Ho <= 0 || Wo <= 0) return -2;
    conv_ctx c = {x, w, bias, y, C, H, W, F, S, stride, pad, groups, relu, Ho, Wo};
    for_each_image(conv_item, &c, B * F, nthreads);
    return 0;
}

/* Fig. 2 literally: step 1 im2col -> D_m, step 2 F_m, step 3 F_m x D_m. */
int orc_conv2d_im2col_gemm(const double *x, int B, int C, int H, int W,
                           const double *w, const double *bias, int F, int S,
                           int stride, int pad, int groups, int relu,
                           double *y) {
    if (!x || !w || !y || groups <= 0 || C % groups || F % groups) return -1;
    const int Ho = orc_conv_out_size(H, S, stride, pad);
    const int Wo = orc_conv_out_size(W, S, stride, pad);
    if (Ho <= 0 || Wo <= 0) return -2;
    const int Cg = C / groups, Fg = F / groups;
    const size_t Kd = (size_t)S * S * Cg, P = (size_t)Ho * Wo;
    double *Dm = (double *)malloc(sizeof(double) * Kd * P);
    if (!Dm) return -3;
    for (int n = 0; n < B; ++n) {
        for (int g = 0; g < groups; ++g) {
            /* step 1: D_m[(c,r,s)][(p,q)] */
            for (int ci = 0; ci < Cg; ++ci)
                for (int r = 0; r < S; ++r)
                    for (int s = 0; s < S; ++s) {
                        const size_t row = ((size_t)ci * S + r) * S + s;
                        for (int p = 0; p < Ho; ++p)
                            for (int q = 0; q < Wo; ++q) {
                                const int ih = p * stride + r - pad;
                                const int iw = q * stride + s - pad;
                                double v = 0.0;
                                if (ih >= 0 && ih < H && iw >= 0 && iw < W)
                                    v = x[(((size_t)n * C + g * Cg + ci) * H + ih) * W + iw];
                                Dm[row * P + (size_t)p * Wo + q] = v;
                            }
                    }
            /* steps 2-3: O_m = F_m x D_m, F_m row f = OIHW weights of filter f */
            for (int fl = 0; fl < Fg; ++fl) {
                const int f = g * Fg + fl;
                const double *Fm = w + (size_t)f * Kd;
                for (size_t pq = 0; pq < P; ++pq) {
                    double acc = 0.0;
                    for (size_t k = 0; k < Kd; ++k) acc += Fm[k] * Dm[k * P + pq];
                    double v = acc + (bias ? bias[f] : 0.0);
                    if (relu && v < 0.0) v = 0.0;
                    y[((size_t)n * F + f) * P + pq] = v;
                }
            }
        }
    }
    free(Dm);
    return 0;
}

/* ------------------------------------------------------------------ */
/* LRN across channels (reading R3, Caffe bvlc_alexnet norm1/norm2)    */
/* ------------------------------------------------------------------ */
typedef struct {
    const double *x;
    double *y;
    int C, H, W, size;
    double alpha, beta, k;
} lrn_ctx;

static void lrn_image(void *vctx, int n) {
    const lrn_ctx *c = (const lrn_ctx *)vctx;
    const int half = c->size / 2;
    const size_t HW = (size_t)c->H * c->W;
    for (int ch = 0; ch < c->C; ++ch) {
        int lo = ch - half, hi = ch + half;
        if (lo < 0) lo = 0;
        if (hi > c->C - 1) hi = c->C - 1;
        for (size_t i = 0; i < HW; ++i) {
            double sq = 0.0;
            for (int cc = lo; cc <= hi; ++cc) {
                const double a = c->x[((size_t)n * c->C + cc) * HW + i];
                sq += a * a;
            }
            const double scale = c->k + c->alpha / c->size * sq;
            c->y[((size_t)n * c->C + ch) * HW + i] =
                c->x[((size_t)n * c->C + ch) * HW + i] / pow(scale, c->beta);
        }
    }
}

int orc_lrn(const double *x, int B, int C, int H, int W, int size,
            double alpha, double beta, double k, double *y, int nthreads) {
    if (!x || !y || size <= 0 || (size % 2) == 0) return -1;
    lrn_ctx c = {x, y, C, H, W, size, alpha, beta, k};
    for_each_image(lrn_image, &c, B, nthreads);
    return 0;
}

/* ------------------------------------------------------------------ */
/* pooling ("max-pooling layers")                                 */
/* ------------------------------------------------------------------ */
typedef struct {
    const double *x;
    double *y;
    int C, H, W, k, stride, Ho, Wo, is_max;
} pool_ctx;

static void pool_image(void *vctx, int n) {
    const pool_ctx *c = (const pool_ctx *)vctx;
    for (int ch = 0; ch < c->C; ++ch)
        for (int p = 0; p < c->Ho; ++p)
            for (int q = 0; q < c->Wo; ++q) {
                int h0 = p * c->stride, w0 = q * c->stride;
                int h1 = h0 + c->k, w1 = w0 + c->k;
                if (h1 > c->H) h1 = c->H;
                if (w1 > c->W) w1 = c->W;
                double m = -INFINITY, s = 0.0;
                for (int h = h0; h < h1; ++h)
                    for (int w = w0; w < w1; ++w) {
                        const double v = c->x[(((size_t)n * c->C + ch) * c->H + h) * c->W + w];
                        if (v > m) m = v;
                        s += v;
                    }
                c->y[(((size_t)n * c->C + ch) * c->Ho + p) * c->Wo + q] =
                    c->is_max ? m : s / ((double)c->k * c->k);
            }
}

static int pool_common(const double *x, int B, int C, int H, int W, int k,
                       int stride, double *y, int nthreads, int is_max) {
    if (!x || !y || k <= 0) return -1;
    int Ho = orc_pool_out_size(H, k, stride), Wo = orc_pool_out_size(W, k, stride);
    if (Ho <= 0 || Wo <= 0) return -2;
    pool_ctx c = {x, y, C, H, W, k, stride, Ho, Wo, is_max};
    for_each_image(pool_image, &c, B, nthreads);
    return 0;
}

int orc_maxpool(const double *x, int B, int C, int H, int W, int k,
                int stride, double *y, int nthreads) {
    return pool_common(x, B, C, H, W, k, stride, y, nthreads, 1);
}

int orc_avgpool(const double *x, int B, int C, int H, int W, int k,
                int stride, double *y, int nthreads) {
    return pool_common(x, B, C, H, W, k, stride, y, nthreads, 0);
}

/* ------------------------------------------------------------------ */
/* classifier (FC) layer                                               */
/* ------------------------------------------------------------------ */
typedef struct {
    const double *x, *w, *bias;
    double *y;
    int K, N, relu;
} fc_ctx;

/* one work item = one output feature j of one image n */
static void fc_item(void *vctx, int item) {
    const fc_ctx *c = (const fc_ctx *)vctx;
    const int n = item / c->N, j = item % c->N;
    double acc = 0.0;
    for (int i = 0; i < c->K; ++i)
        acc += c->w[(size_t)j * c->K + i] * c->x[(size_t)n * c->K + i];
    double v = acc + (c->bias ? c->bias[j] : 0.0);
    if (c->relu && v < 0.0) v = 0.0;
    c->y[(size_t)n * c->N + j] = v;
}

int orc_fc(const double *x, int B, int K, const double *w, const double *bias,
           int N, int relu, double *y, int nthreads) {
    if (!x || !w || !y || K <= 0 || N <= 0) return -1;
    fc_ctx c = {x, w, bias, y, K, N, relu};
    for_each_image(fc_item, &c, B * N, nthreads);
    return 0;
}

/* ------------------------------------------------------------------ */
/* softmax + entropy (eq. 2)                           */
/* ------------------------------------------------------------------ */
double orc_entropy(const double *p, int n) {
    double h = 0.0;
    for (int i = 0; i < n; ++i)
        if (p[i] > 0.0) h -= p[i] * log(p[i]);      /* 0 ln 0 = 0 */
    return h;
}

int orc_softmax_entropy(const double *z, int B, int N, double *p, double *H) {
    if (!z || N <= 0) return -1;
    double *tmp = p ? NULL : (double *)malloc(sizeof(double) * (size_t)N);
    for (int n = 0; n < B; ++n) {
        const double *zr = z + (size_t)n * N;
        double *pr = p ? p + (size_t)n * N : tmp;
        double m = zr[0];
        for (int j = 1; j < N; ++j) if (zr[j] > m) m = zr[j];
        double s = 0.0;
        for (int j = 0; j < N; ++j) { pr[j] = exp(zr[j] - m); s += pr[j]; }
        for (int j = 0; j < N; ++j) pr[j] /= s;
        if (H) H[n] = orc_entropy(pr, N);
    }
    free(tmp);
    return 0;
}

/* ------------------------------------------------------------------ */
/* rank-r operator via the Gram matrix (reading R7)                    */
/* ------------------------------------------------------------------ */
/* Cyclic Jacobi eigen-decomposition of a symmetric n x n matrix A
 * (overwritten).  V receives the eigenvectors as columns. */
static void jacobi_eigen(double *A, int n, double *V) {
    for (int i = 0; i < n; ++i)
        for (int j = 0; j < n; ++j) V[(size_t)i * n + j] = (i == j) ? 1.0 : 0.0;
    for (int sweep = 0; sweep < 100; ++sweep) {
        double off = 0.0, diag = 0.0;
        for (int i = 0; i < n; ++i) {
            diag += A[(size_t)i * n + i] * A[(size_t)i * n + i];
            for (int j = i + 1; j < n; ++j) off += A[(size_t)i * n + j] * A[(size_t)i * n + j];
        }
        if (off <= 1e-26 * diag || off == 0.0) break;
        for (int p = 0; p < n - 1; ++p)
            for (int q = p + 1; q < n; ++q) {
                const double apq = A[(size_t)p * n + q];
                const double app = A[(size_t)p * n + p], aqq = A[(size_t)q * n + q];
                if (fabs(apq) <= 1e-18 * (fabs(app) + fabs(aqq)) || fabs(apq) < 1e-300) continue;
                const double theta = (aqq - app) / (2.0 * apq);
                const double t = (theta >= 0 ? 1.0 : -1.0) /
                                 (fabs(theta) + sqrt(theta * theta + 1.0));
                const double cs = 1.0 / sqrt(t * t + 1.0), sn = t * cs;
                for (int k = 0; k < n; ++k) {          /* A <- A J (columns p,q) */
                    const double akp = A[(size_t)k * n + p], akq = A[(size_t)k * n + q];
                    A[(size_t)k * n + p] = cs * akp - sn * akq;
                    A[(size_t)k * n + q] = sn * akp + cs * akq;
                }
                for (int k = 0; k < n; ++k) {          /* A <- J^T A (rows p,q) */
                    const double apk = A[(size_t)p * n + k], aqk = A[(size_t)q * n + k];
                    A[(size_t)p * n + k] = cs * apk - sn * aqk;
                    A[(size_t)q * n + k] = sn * apk + cs * aqk;
                }
                for (int k = 0; k < n; ++k) {          /* V <- V J */
                    const double vkp = V[(size_t)k * n + p], vkq = V[(size_t)k * n + q];
                    V[(size_t)k * n + p] = cs * vkp - sn * vkq;
                    V[(size_t)k * n + q] = sn * vkp + cs * vkq;
                }
            }
    }
}

int orc_rank_r(const double *Wm, int N, int K, int r, double *Wr, double *sigma) {
    if (!Wm || !Wr || N <= 0 || K <= 0 || r < 0) return -1;
    const int mn = N < K ? N : K;
    if (r > mn) r = mn;
    double *G = (double *)malloc(sizeof(double) * (size_t)N * N);
    double *V = (double *)malloc(sizeof(double) * (size_t)N * N);
    int *order = (int *)malloc(sizeof(int) * (size_t)N);
    if (!G || !V || !order) { free(G); free(V); free(order); return -3; }
    /* G = Wm Wm^T */
    for (int i = 0; i < N; ++i)
        for (int j = 0; j < N; ++j) {
            double s = 0.0;
            for (int k = 0; k < K; ++k) s += Wm[(size_t)i * K + k] * Wm[(size_t)j * K + k];
            G[(size_t)i * N + j] = s;
        }
    jacobi_eigen(G, N, V);
    /* order eigenvalues descending (selection sort: N <= a few hundred) */
    for (int i = 0; i < N; ++i) order[i] = i;
    for (int i = 0; i < N; ++i) {
        int best = i;
        for (int j = i + 1; j < N; ++j)
            if (G[(size_t)order[j] * N + order[j]] > G[(size_t)order[best] * N + order[best]]) best = j;
        int t = order[i]; order[i] = order[best]; order[best] = t;
    }
    double s1 = 0.0, sr = 0.0, sr1 = 0.0;
    for (int i = 0; i < mn; ++i) {
        double lam = G[(size_t)order[i] * N + order[i]];
        double sv = lam > 0.0 ? sqrt(lam) : 0.0;
        if (sigma) sigma[i] = sv;
        if (i == 0) s1 = sv;
        if (i == r - 1) sr = sv;
        if (i == r) sr1 = sv;
    }
    /* W_r = U_r U_r^T Wm */
    double *T = (double *)calloc((size_t)r * K + 1, sizeof(double));  /* U_r^T Wm, r x K */
    if (!T) { free(G); free(V); free(order); return -3; }
    for (int a = 0; a < r; ++a) {
        const int col = order[a];
        for (int k = 0; k < K; ++k) {
            double s = 0.0;
            for (int i = 0; i < N; ++i) s += V[(size_t)i * N + col] * Wm[(size_t)i * K + k];
            T[(size_t)a * K + k] = s;
        }
    }
    for (int i = 0; i < N; ++i)
        for (int k = 0; k < K; ++k) {
            double s = 0.0;
            for (int a = 0; a < r; ++a) s += V[(size_t)i * N + order[a]] * T[(size_t)a * K + k];
            Wr[(size_t)i * K + k] = s;
        }
    free(T); free(G); free(V); free(order);
    if (r > 0 && r < mn && s1 > 0.0 && (sr - sr1) / s1 < 1e-6) return 1;
    return 0;
}

/* ------------------------------------------------------------------ */
/* analytical helpers                           */
/* ------------------------------------------------------------------ */
static long cdiv(long a, long b) { return (a + b - 1) / b; }

long orc_grid_size(long M, long N, long m, long n) {           /* eq. 4 */
    return cdiv(M, m) * cdiv(N, n);
}
long orc_max_blocks(long nSMs, long R, long block_size, long r) { /* eq. 5 */
    return nSMs * (R / (block_size * r));
}
double orc_util(long grid, long max_blocks) {                   /* eq. 6, reading R8 */
    return (double)grid / ((double)cdiv(grid, max_blocks) * (double)max_blocks);
}
long orc_n_invocations(long grid, long tlp, long nSMs) {         /* eq. 8 */
    return cdiv(grid, tlp * nSMs);
}
double orc_rec(long M, long N, long m, long n) {                /* eq. 9 */
    return (double)M * (double)N / ((double)cdiv(M, m) * cdiv(N, n) * m * n);
}
long orc_opt_sm(long grid, long opt_tlp, long num_sms) {         /* eq. 11 */
    const long target = cdiv(grid, opt_tlp * num_sms);
    for (long s = 1; s <= num_sms; ++s)
        if (cdiv(grid, opt_tlp * s) == target) return s;
    return num_sms;
}
