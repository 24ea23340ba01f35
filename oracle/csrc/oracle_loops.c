/*
 * oracle_loops.c -- TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).
 *
 * Plain direct loops for ONE patch of a Split-CNN window operator, in fp64.
 * Every loop is the textbook definition written out; there is no blocking,
 * no im2col, no reordering beyond the formula.  Layout is the paper's
 * logical NCHW for each patch X_n = Split_W(X, I)[n] (Eq. 4).
 *
 * The per-patch operator is Y_n = Op(X_n, k, s, p_n) (Eq. 6):
 * an ordinary convolution / max-pool of the separately padded patch.  The
 * begin pads (pt, pl) enter as "h = oh*s - pt + r"; the end pads are implied
 * by the output extent Ho, Wo that the caller computes from them.
 *
 * Shares no code with the CUDA path (paper_conf_asplos_jinh19_b200/csrc).
 */
#include <math.h>
#include <stddef.h>

#define IDX4(a, b, c, d, B, C, D) ((((size_t)(a) * (B) + (b)) * (C) + (c)) * (D) + (d))

/* O3: conv forward of one patch (Eq. 6).
 * Y[n,co,oh,ow] = bias[co] + sum_{ci,r,c} X[n,ci,oh*sh-pt+r, ow*sw-pl+c] * W[co,ci,r,c],
 * taps outside the patch read the zero padding; then ReLU if relu != 0. */
void oracle_conv_fwd(const double *X, const double *W, const double *bias, double *Y,
                     int N, int Ci, int Hp, int Wp, int Co, int kh, int kw, int sh, int sw,
                     int pt, int pl, int Ho, int Wo, int relu)
{
    #pragma omp parallel for collapse(2) schedule(static)
    for (int n = 0; n < N; ++n)
        for (int co = 0; co < Co; ++co)
            for (int oh = 0; oh < Ho; ++oh)
                for (int ow = 0; ow < Wo; ++ow) {
                    double acc = bias ? bias[co] : 0.0;
                    for (int ci = 0; ci < Ci; ++ci)
                        for (int r = 0; r < kh; ++r)
                            for (int c = 0; c < kw; ++c) {
                                int h = oh * sh - pt + r;
                                int w = ow * sw - pl + c;
                                if (h >= 0 && h < Hp && w >= 0 && w < Wp)
                                    acc += X[IDX4(n, ci, h, w, Ci, Hp, Wp)] *
                                           W[IDX4(co, ci, r, c, Ci, kh, kw)];
                            }
                    if (relu && acc < 0.0) acc = 0.0;
                    Y[IDX4(n, co, oh, ow, Co, Ho, Wo)] = acc;
                }
}

/* O4: conv data gradient of one patch (adjoint of Eq. 6).
 * dX[n,ci,h,w] = sum over co, r, c with oh = (h+pt-r)/sh integral and in [0,Ho)
 * (same for w) of dY[n,co,oh,ow] * W[co,ci,r,c].  The gradient never leaves the
 * patch.  If mask != NULL, dX is multiplied by [mask > 0]
 * (the backward of the ReLU that produced this layer's input). */
void oracle_conv_bwd_data(const double *dY, const double *W, const double *mask, double *dX,
                          int N, int Ci, int Hp, int Wp, int Co, int kh, int kw, int sh, int sw,
                          int pt, int pl, int Ho, int Wo)
{
    #pragma omp parallel for collapse(2) schedule(static)
    for (int n = 0; n < N; ++n)
        for (int ci = 0; ci < Ci; ++ci)
            for (int h = 0; h < Hp; ++h)
                for (int w = 0; w < Wp; ++w) {
                    double acc = 0.0;
                    for (int co = 0; co < Co; ++co)
                        for (int r = 0; r < kh; ++r)
                            for (int c = 0; c < kw; ++c) {
                                int th = h + pt - r, tw = w + pl - c;
                                if (th < 0 || tw < 0 || th % sh != 0 || tw % sw != 0) continue;
                                int oh = th / sh, ow = tw / sw;
                                if (oh >= Ho || ow >= Wo) continue;
                                acc += dY[IDX4(n, co, oh, ow, Co, Ho, Wo)] *
                                       W[IDX4(co, ci, r, c, Ci, kh, kw)];
                            }
                    size_t i = IDX4(n, ci, h, w, Ci, Hp, Wp);
                    if (mask && !(mask[i] > 0.0)) acc = 0.0;
                    dX[i] = acc;
                }
}

/* O5: conv weight gradient contribution of one patch.
 * dW[co,ci,r,c] = sum_{n,oh,ow} dY[n,co,oh,ow] * X~[n,ci,oh*sh-pt+r, ow*sw-pl+c],
 * X~ = 0 outside the patch.  db[co] = sum_{n,oh,ow} dY[n,co,oh,ow] (R12).
 * Written into dW/db (overwrite); the caller sums over patches. */
void oracle_conv_bwd_filter(const double *X, const double *dY, double *dW, double *db,
                            int N, int Ci, int Hp, int Wp, int Co, int kh, int kw, int sh, int sw,
                            int pt, int pl, int Ho, int Wo)
{
    #pragma omp parallel for collapse(2) schedule(static)
    for (int co = 0; co < Co; ++co)
        for (int ci = 0; ci < Ci; ++ci)
            for (int r = 0; r < kh; ++r)
                for (int c = 0; c < kw; ++c) {
                    double acc = 0.0;
                    for (int n = 0; n < N; ++n)
                        for (int oh = 0; oh < Ho; ++oh)
                            for (int ow = 0; ow < Wo; ++ow) {
                                int h = oh * sh - pt + r;
                                int w = ow * sw - pl + c;
                                if (h >= 0 && h < Hp && w >= 0 && w < Wp)
                                    acc += dY[IDX4(n, co, oh, ow, Co, Ho, Wo)] *
                                           X[IDX4(n, ci, h, w, Ci, Hp, Wp)];
                            }
                    dW[IDX4(co, ci, r, c, Ci, kh, kw)] = acc;
                }
    if (db) {
        for (int co = 0; co < Co; ++co) {
            double acc = 0.0;
            for (int n = 0; n < N; ++n)
                for (int oh = 0; oh < Ho; ++oh)
                    for (int ow = 0; ow < Wo; ++ow)
                        acc += dY[IDX4(n, co, oh, ow, Co, Ho, Wo)];
            db[co] = acc;
        }
    }
}

/* O6: max-pool forward of one patch (readings R7-R9).
 * Y = max over the in-patch window elements (padding is -inf, i.e. skipped);
 * argmax = window-local r*kw+c of the FIRST maximum in row-major window order
 * (strict '>').  An all-padding window cannot occur for pads < k. */
void oracle_pool_fwd(const double *X, double *Y, int *argmax,
                     int N, int C, int Hp, int Wp, int kh, int kw, int sh, int sw,
                     int pt, int pl, int Ho, int Wo)
{
    #pragma omp parallel for collapse(2) schedule(static)
    for (int n = 0; n < N; ++n)
        for (int ch = 0; ch < C; ++ch)
            for (int oh = 0; oh < Ho; ++oh)
                for (int ow = 0; ow < Wo; ++ow) {
                    double best = -INFINITY;
                    int arg = -1;
                    for (int r = 0; r < kh; ++r)
                        for (int c = 0; c < kw; ++c) {
                            int h = oh * sh - pt + r;
                            int w = ow * sw - pl + c;
                            if (h < 0 || h >= Hp || w < 0 || w >= Wp) continue;
                            double v = X[IDX4(n, ch, h, w, C, Hp, Wp)];
                            if (arg < 0 || v > best) { best = v; arg = r * kw + c; }
                        }
                    size_t o = IDX4(n, ch, oh, ow, C, Ho, Wo);
                    Y[o] = best;
                    argmax[o] = arg;
                }
}

/* O7: max-pool backward of one patch: dX[argmax] += dY (R10: accumulate). */
void oracle_pool_bwd(const double *dY, const int *argmax, double *dX,
                     int N, int C, int Hp, int Wp, int kh, int kw, int sh, int sw,
                     int pt, int pl, int Ho, int Wo)
{
    #pragma omp parallel for collapse(2) schedule(static)
    for (int n = 0; n < N; ++n)
        for (int ch = 0; ch < C; ++ch) {
            for (int h = 0; h < Hp; ++h)
                for (int w = 0; w < Wp; ++w)
                    dX[IDX4(n, ch, h, w, C, Hp, Wp)] = 0.0;
            for (int oh = 0; oh < Ho; ++oh)
                for (int ow = 0; ow < Wo; ++ow) {
                    size_t o = IDX4(n, ch, oh, ow, C, Ho, Wo);
                    int a = argmax[o];
                    int h = oh * sh - pt + a / kw;
                    int w = ow * sw - pl + a % kw;
                    dX[IDX4(n, ch, h, w, C, Hp, Wp)] += dY[o];
                }
        }
    (void)kh;
}
