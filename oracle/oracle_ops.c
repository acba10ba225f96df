/*
 * ORACLE -- TEST INFRASTRUCTURE ONLY.
 *
 * Plain, slow, obviously-correct fp64 CPU implementation of every layer on the
 * DjiNN hot path (the batched DNN forward pass, sec 3 and L183-185
 * sec 5.1).  Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
 * --impl reference legs may load this library.  It shares no code, header, table or
 * helper with the CUDA path (paper_conf_isca_hauswaldklclmdm15_b200/csrc).
 *
 * Conventions: tensors are dense C-order NCHW (Caffe blobs, "we use
 * Caffe"), fp64, no rounding of activations.  Every reduction is accumulated in the
 * order written, starting from the bias.  OpenMP parallelises over independent
 * output elements only (never splits a sum), so results do not depend on the
 * thread count.
 *
 * Definitions (SURVEY.md sec 8(c) "Per-op definitions"; readings in DESIGN.md sec 3):
 *   conv  : Caffe cross-correlation with zero padding and groups  [PAPER.md L65]
 *   local : unshared ("locally-connected") conv, DeepFace L4-L6    [L100, ext ref 43]
 *   ip    : fully-connected y = W x + b                            [L63]
 *   lrn   : Caffe ACROSS_CHANNELS LRN                              [ext ref 28 @ L392]
 *   pool  : Caffe MAX / AVE pooling, ceil geometry                 [L65]
 *   softmax, relu, sigmoid, tanh, hardtanh                         [L55, L92]
 */
#include <math.h>
#include <float.h>
#include <stdint.h>
#include <stdlib.h>

#define IDX4(n, c, h, w, C, H, W) ((((int64_t)(n) * (C) + (c)) * (H) + (h)) * (W) + (w))

int orc_version(void) { return 1; }

/* Output size of a convolution / locally-connected layer (Caffe floor formula). */
int orc_conv_out(int in, int k, int s, int p) { return (in + 2 * p - k) / s + 1; }

/* Output size of a pooling layer (Caffe ceil formula, with the pad correction). */
int orc_pool_out(int in, int k, int s, int p) {
    int out = (int)ceil((double)(in + 2 * p - k) / (double)s) + 1;
    if (p > 0 && (int64_t)(out - 1) * s >= in + p) --out;
    return out;
}

/*
 * y[n,co,oy,ox] = b[co] + sum_{ci<C/g} sum_{ky<KH} sum_{kx<KW}
 *                 w[co,ci,ky,kx] * x[n, g*C/g + ci, oy*s-p+ky, ox*s-p+kx]
 * with g = co / (Co/g); x is 0 outside [0,H)x[0,W).
 * w: [Co, C/group, KH, KW], b: [Co], y: [N, Co, OH, OW].
 */
void orc_conv2d(const double* x, int N, int C, int H, int W,
                const double* w, const double* b, int Co, int KH, int KW,
                int stride, int pad, int group, double* y) {
    const int OH = orc_conv_out(H, KH, stride, pad), OW = orc_conv_out(W, KW, stride, pad);
    const int Cg = C / group, Cog = Co / group;
    #pragma omp parallel for collapse(2) schedule(dynamic)
    for (int n = 0; n < N; ++n)
        for (int co = 0; co < Co; ++co) {
            const int g = co / Cog;
            double* acc = (double*)malloc(sizeof(double) * OW);
            for (int oy = 0; oy < OH; ++oy) {
                for (int ox = 0; ox < OW; ++ox) acc[ox] = b[co];
                for (int ci = 0; ci < Cg; ++ci)
                    for (int ky = 0; ky < KH; ++ky) {
                        const int iy = oy * stride - pad + ky;
                        if (iy < 0 || iy >= H) continue;
                        const double* xr = x + IDX4(n, g * Cg + ci, iy, 0, C, H, W);
                        for (int kx = 0; kx < KW; ++kx) {
                            const double wv = w[IDX4(co, ci, ky, kx, Cg, KH, KW)];
                            for (int ox = 0; ox < OW; ++ox) {   /* independent sums, one per ox */
                                const int ix = ox * stride - pad + kx;
                                if (ix >= 0 && ix < W) acc[ox] += wv * xr[ix];
                            }
                        }
                    }
                for (int ox = 0; ox < OW; ++ox) y[IDX4(n, co, oy, ox, Co, OH, OW)] = acc[ox];
            }
            free(acc);
        }
}

/*
 * Locally-connected (unshared weights), no padding:
 * y[n,co,oy,ox] = b[co,oy,ox] + sum_{ci,ky,kx} w[oy,ox,co,ci,ky,kx] * x[n,ci,oy*s+ky,ox*s+kx]
 * w: [OH, OW, Co, C, KH, KW] (one Caffe-style filter bank per output location),
 * b: [Co, OH, OW], y: [N, Co, OH, OW].
 */
void orc_local(const double* x, int N, int C, int H, int W,
               const double* w, const double* b, int Co, int KH, int KW, int stride, double* y) {
    const int OH = orc_conv_out(H, KH, stride, 0), OW = orc_conv_out(W, KW, stride, 0);
    #pragma omp parallel for collapse(2) schedule(dynamic)
    for (int n = 0; n < N; ++n)
        for (int co = 0; co < Co; ++co)
            for (int oy = 0; oy < OH; ++oy)
                for (int ox = 0; ox < OW; ++ox) {
                    const double* wl = w + ((((int64_t)oy * OW + ox) * Co + co) * C) * KH * KW;
                    double acc = b[((int64_t)co * OH + oy) * OW + ox];
                    for (int ci = 0; ci < C; ++ci)
                        for (int ky = 0; ky < KH; ++ky)
                            for (int kx = 0; kx < KW; ++kx)
                                acc += wl[((int64_t)ci * KH + ky) * KW + kx] *
                                       x[IDX4(n, ci, oy * stride + ky, ox * stride + kx, C, H, W)];
                    y[IDX4(n, co, oy, ox, Co, OH, OW)] = acc;
                }
}

/* y[n,o] = b[o] + sum_k w[o,k] * x[n,k];  x: [N,K] (Caffe flattens (c,h,w)), w: [No,K]. */
void orc_inner_product(const double* x, int N, int K, const double* w, const double* b,
                       int No, double* y) {
    #pragma omp parallel for collapse(2) schedule(static)
    for (int n = 0; n < N; ++n)
        for (int o = 0; o < No; ++o) {
            const double* xr = x + (int64_t)n * K;
            const double* wr = w + (int64_t)o * K;
            double acc = b[o];
            for (int k = 0; k < K; ++k) acc += wr[k] * xr[k];
            y[(int64_t)n * No + o] = acc;
        }
}

/* Element-wise activations, in place (Caffe ReLU with negative_slope 0, Sigmoid, TanH;
 * SENNA HardTanh = clamp to [-1, 1]). */
void orc_relu(double* x, int64_t n) {
    #pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < n; ++i) x[i] = x[i] > 0.0 ? x[i] : 0.0;
}
void orc_sigmoid(double* x, int64_t n) {
    #pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < n; ++i) x[i] = 1.0 / (1.0 + exp(-x[i]));
}
void orc_tanh(double* x, int64_t n) {
    #pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < n; ++i) x[i] = tanh(x[i]);
}
void orc_hardtanh(double* x, int64_t n) {
    #pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < n; ++i) x[i] = x[i] < -1.0 ? -1.0 : (x[i] > 1.0 ? 1.0 : x[i]);
}

/*
 * Caffe LRN, ACROSS_CHANNELS:
 * y[n,c,h,w] = x[n,c,h,w] * ( k + alpha/size * sum_{c'=max(0,c-(size-1)/2)}^{min(C-1,c+(size-1)/2)} x[n,c',h,w]^2 )^(-beta)
 */
void orc_lrn(const double* x, int N, int C, int H, int W, int size, double alpha,
             double beta, double k, double* y) {
    const int half = (size - 1) / 2;
    #pragma omp parallel for collapse(2) schedule(static)
    for (int n = 0; n < N; ++n)
        for (int c = 0; c < C; ++c) {
            const int lo = c - half < 0 ? 0 : c - half;
            const int hi = c + half > C - 1 ? C - 1 : c + half;
            for (int h = 0; h < H; ++h)
                for (int w = 0; w < W; ++w) {
                    double s = 0.0;
                    for (int cc = lo; cc <= hi; ++cc) {
                        const double v = x[IDX4(n, cc, h, w, C, H, W)];
                        s += v * v;
                    }
                    const double scale = k + alpha / size * s;
                    y[IDX4(n, c, h, w, C, H, W)] = x[IDX4(n, c, h, w, C, H, W)] * pow(scale, -beta);
                }
        }
}

/*
 * Caffe pooling.  Window rows [oy*s - p, min(oy*s - p + k, H + p)), clipped to [0, H)
 * (same for columns).  MAX: maximum over the clipped window.  AVE: sum over the clipped
 * window divided by the window area computed BEFORE clipping to [0,H) but after
 * clipping to H+p.  mode: 0 = MAX, 1 = AVE.
 */
void orc_pool(const double* x, int N, int C, int H, int W, int mode, int kh, int kw,
              int stride, int pad, double* y) {
    const int OH = orc_pool_out(H, kh, stride, pad), OW = orc_pool_out(W, kw, stride, pad);
    #pragma omp parallel for collapse(2) schedule(static)
    for (int n = 0; n < N; ++n)
        for (int c = 0; c < C; ++c)
            for (int oy = 0; oy < OH; ++oy)
                for (int ox = 0; ox < OW; ++ox) {
                    int hs = oy * stride - pad, ws = ox * stride - pad;
                    int he = hs + kh < H + pad ? hs + kh : H + pad;
                    int we = ws + kw < W + pad ? ws + kw : W + pad;
                    const double area = (double)(he - hs) * (double)(we - ws);
                    if (hs < 0) hs = 0;
                    if (ws < 0) ws = 0;
                    if (he > H) he = H;
                    if (we > W) we = W;
                    double r;
                    if (mode == 0) {
                        r = -DBL_MAX;
                        for (int h = hs; h < he; ++h)
                            for (int w = ws; w < we; ++w) {
                                const double v = x[IDX4(n, c, h, w, C, H, W)];
                                if (v > r) r = v;
                            }
                    } else {
                        r = 0.0;
                        for (int h = hs; h < he; ++h)
                            for (int w = ws; w < we; ++w) r += x[IDX4(n, c, h, w, C, H, W)];
                        r /= area;
                    }
                    y[IDX4(n, c, oy, ox, C, OH, OW)] = r;
                }
}

/* Row softmax, stable form: p_i = exp(z_i - max z) / sum_j exp(z_j - max z). */
void orc_softmax(const double* x, int N, int D, double* y) {
    #pragma omp parallel for schedule(static)
    for (int n = 0; n < N; ++n) {
        const double* z = x + (int64_t)n * D;
        double* p = y + (int64_t)n * D;
        double m = z[0];
        for (int i = 1; i < D; ++i) if (z[i] > m) m = z[i];
        double s = 0.0;
        for (int i = 0; i < D; ++i) { p[i] = exp(z[i] - m); s += p[i]; }
        for (int i = 0; i < D; ++i) p[i] /= s;
    }
}

/* Row argmax; ties resolve to the lowest index. */
void orc_argmax(const double* x, int N, int D, int32_t* out) {
    for (int n = 0; n < N; ++n) {
        const double* z = x + (int64_t)n * D;
        int best = 0;
        for (int i = 1; i < D; ++i) if (z[i] > z[best]) best = i;
        out[n] = best;
    }
}
