/*
 * otif_ref_train.c — CPU ORACLE for NEXT-3, proxy training labels and training
 * (P:L137–141).
 *
 * TEST INFRASTRUCTURE ONLY (see otif_ref.h).  Plain C99 in fp64, no quantisation:
 *   labels  "at each 32 x 32 cell, the label is 1 if there is some detection d_i in D(t)
 *           that intersects the cell, and 0 otherwise";
 *   loss    "the model should output a score close to 1 at cells that intersect a
 *           detection, and 0 at other cells": binary cross-entropy on
 *           score = sigmoid(z), averaged over the cells of the batch (reading R26);
 *   grads   backpropagation through D2, D1, E5..E1 written out per layer (chain rule,
 *           no fusion): ReLU passes the gradient where its output is positive;
 *   update  Adam (reading R27).
 * The forward pass is otif_ref_conv (the inference oracle's convolution) with quant=none.
 */
#include "otif_ref.h"

#include <math.h>
#include <stdlib.h>
#include <string.h>

/* ------------------------------------------------------------------------- */
/* P:L139 labels.  Cell (cy, cx) covers [cx·cell, min((cx+1)·cell, W)) x [cy·cell, ...)
 * (reading R14); a detection [x0, x1) x [y0, y1) intersects it when the open
 * rectangles overlap.  boxes int32 [nb][5] = (frame, x0, y0, x1, y1). */
int otif_ref_cell_labels(const int32_t *boxes, int64_t nb, int32_t n, int32_t gh, int32_t gw, int32_t cell,
                         int32_t frame_w, int32_t frame_h, uint8_t *labels) {
    if (n < 0 || gh <= 0 || gw <= 0 || cell <= 0) return -1;
    memset(labels, 0, (size_t)n * gh * gw);
    for (int32_t f = 0; f < n; f++)
        for (int32_t cy = 0; cy < gh; cy++)
            for (int32_t cx = 0; cx < gw; cx++) {
                int32_t ax0 = cx * cell, ay0 = cy * cell;
                int32_t ax1 = (cx + 1) * cell < frame_w ? (cx + 1) * cell : frame_w;
                int32_t ay1 = (cy + 1) * cell < frame_h ? (cy + 1) * cell : frame_h;
                for (int64_t b = 0; b < nb; b++) {
                    const int32_t *d = boxes + 5 * b;
                    if (d[0] != f) continue;
                    if (d[1] >= d[3] || d[2] >= d[4]) continue;   /* an empty box intersects nothing */
                    if (d[1] < ax1 && ax0 < d[3] && d[2] < ay1 && ay0 < d[4]) {
                        labels[((size_t)f * gh + cy) * gw + cx] = 1;
                        break;
                    }
                }
            }
    return 0;
}

/* ------------------------------------------------------------------------- */
/* Backward of one convolution y = conv(x, W) + b (pad (k−1)/2, stride s), given
 * dy = ∂L/∂y (the gradient at the convolution's output, before any activation):
 *   dx[f, iy, ix, ci]      = Σ_{co, kh, kw : iy = s·oy − pad + kh, ix = s·ox − pad + kw} dy[f, oy, ox, co] · W[co, kh, kw, ci]
 *   dW[co, kh, kw, ci]     = Σ_{f, oy, ox} dy[f, oy, ox, co] · x[f, s·oy − pad + kh, s·ox − pad + kw, ci]
 *   db[co]                 = Σ_{f, oy, ox} dy[f, oy, ox, co]
 * dx may be NULL.  dW/db are overwritten. */
int otif_ref_conv_backward(const double *x, int32_t n, int32_t h, int32_t w, int32_t cin, const double *weight,
                           int32_t cout, int32_t k, int32_t stride, const double *dy, double *dx, double *dW,
                           double *db) {
    if (n < 0 || h <= 0 || w <= 0 || cin <= 0 || cout <= 0) return -1;
    if (!(k == 1 || k == 3) || !(stride == 1 || stride == 2)) return -1;
    int32_t pad = (k - 1) / 2;
    int32_t ho = (h + stride - 1) / stride, wo = (w + stride - 1) / stride;
    if (dx) memset(dx, 0, sizeof(double) * (size_t)n * h * w * cin);
    memset(dW, 0, sizeof(double) * (size_t)cout * k * k * cin);
    memset(db, 0, sizeof(double) * (size_t)cout);
    for (int32_t f = 0; f < n; f++)
        for (int32_t oy = 0; oy < ho; oy++)
            for (int32_t ox = 0; ox < wo; ox++) {
                const double *g = dy + (((size_t)f * ho + oy) * wo + ox) * cout;
                for (int32_t co = 0; co < cout; co++) {
                    db[co] += g[co];
                    for (int32_t kh = 0; kh < k; kh++) {
                        int32_t iy = stride * oy - pad + kh;
                        if (iy < 0 || iy >= h) continue;
                        for (int32_t kw = 0; kw < k; kw++) {
                            int32_t ix = stride * ox - pad + kw;
                            if (ix < 0 || ix >= w) continue;
                            const double *xi = x + (((size_t)f * h + iy) * w + ix) * cin;
                            const double *wt = weight + (((size_t)co * k + kh) * k + kw) * cin;
                            double *dwt = dW + (((size_t)co * k + kh) * k + kw) * cin;
                            double *dxi = dx ? dx + (((size_t)f * h + iy) * w + ix) * cin : NULL;
                            for (int32_t ci = 0; ci < cin; ci++) {
                                dwt[ci] += g[co] * xi[ci];
                                if (dxi) dxi[ci] += g[co] * wt[ci];
                            }
                        }
                    }
                }
            }
    return 0;
}

/* ------------------------------------------------------------------------- */
/* P:L137–139 one training example batch: forward (fp64, quant=none), loss, gradient.
 * weights / grad: fp64 blob in the proxy layout (E1..E5, D1, D2; W[Cout][kh][kw][Cin]
 * then b[Cout]).  Reading R26: L = (1/M) Σ_cells [softplus(z) − y·z] (= BCE of
 * sigmoid(z) vs the 0/1 label y), M = n·gh·gw, so ∂L/∂z = (sigmoid(z) − y)/M. */
int otif_ref_proxy_grad(const uint8_t *img, int32_t n, int32_t in_h, int32_t in_w, int32_t n_strided,
                        const int32_t enc[5], int32_t dec, const double *weights, const uint8_t *labels,
                        double *loss, double *grad) {
    int32_t gh, gw;
    if (n <= 0 || otif_ref_proxy_grid(in_h, in_w, n_strided, &gh, &gw)) return -1;
    int32_t cin[7], cout[7], ks[7], hs[8], ws[8], st[7];
    size_t woff[7];
    {
        int32_t c = 3;
        for (int i = 0; i < 5; i++) { cin[i] = c; cout[i] = enc[i]; ks[i] = 3; c = enc[i]; }
        cin[5] = c;   cout[5] = dec; ks[5] = 3;
        cin[6] = dec; cout[6] = 1;   ks[6] = 1;
    }
    hs[0] = in_h; ws[0] = in_w;
    size_t off = 0;
    for (int L = 0; L < 7; L++) {
        st[L] = (L < 5 && L < n_strided) ? 2 : 1;
        hs[L + 1] = (hs[L] + st[L] - 1) / st[L];
        ws[L + 1] = (ws[L] + st[L] - 1) / st[L];
        woff[L] = off;
        off += (size_t)cout[L] * ks[L] * ks[L] * cin[L] + cout[L];
    }
    /* forward: act[0] = (u − 128)/128, act[L+1] = ReLU(conv) for L < 6, act[7] = z */
    double *act[8];
    act[0] = (double *)malloc(sizeof(double) * (size_t)n * in_h * in_w * 3);
    for (size_t i = 0; i < (size_t)n * in_h * in_w * 3; i++) act[0][i] = ((double)img[i] - 128.0) / 128.0;
    for (int L = 0; L < 7; L++) {
        act[L + 1] = (double *)malloc(sizeof(double) * (size_t)n * hs[L + 1] * ws[L + 1] * cout[L]);
        const double *wt = weights + woff[L];
        const double *bs = wt + (size_t)cout[L] * ks[L] * ks[L] * cin[L];
        otif_ref_conv(act[L], n, hs[L], ws[L], cin[L], wt, bs, cout[L], ks[L], st[L], L < 6, 0, act[L + 1]);
    }
    /* loss and ∂L/∂z */
    size_t M = (size_t)n * gh * gw;
    double *g = (double *)malloc(sizeof(double) * M);
    double sum = 0.0;
    for (size_t i = 0; i < M; i++) {
        double z = act[7][i], y = labels[i] ? 1.0 : 0.0;
        double softplus = z > 0 ? z + log1p(exp(-z)) : log1p(exp(z));
        sum += softplus - y * z;
        g[i] = (1.0 / (1.0 + exp(-z)) - y) / (double)M;
    }
    *loss = sum / (double)M;
    /* backward, D2 -> E1 */
    for (int L = 6; L >= 0; L--) {
        double *dW = grad + woff[L];
        double *db = dW + (size_t)cout[L] * ks[L] * ks[L] * cin[L];
        size_t nin = (size_t)n * hs[L] * ws[L] * cin[L];
        double *dx = L > 0 ? (double *)malloc(sizeof(double) * nin) : NULL;
        otif_ref_conv_backward(act[L], n, hs[L], ws[L], cin[L], weights + woff[L], cout[L], ks[L], st[L], g, dx, dW,
                               db);
        free(g);
        g = dx;
        if (L > 0) /* act[L] = ReLU(pre): the gradient passes where the output is positive */
            for (size_t i = 0; i < nin; i++)
                if (!(act[L][i] > 0.0)) g[i] = 0.0;
    }
    for (int L = 0; L < 8; L++) free(act[L]);
    return 0;
}

/* ------------------------------------------------------------------------- */
/* Reading R27: Adam (Kingma & Ba), step t >= 1:
 *   m = b1·m + (1 − b1)·g;  v = b2·v + (1 − b2)·g²;
 *   w = w − lr · (m / (1 − b1^t)) / (sqrt(v / (1 − b2^t)) + eps).                  */
int otif_ref_adam(double *w, double *m, double *v, const double *g, int64_t count, int32_t t, double lr, double b1,
                  double b2, double eps) {
    if (count < 0 || t < 1) return -1;
    double c1 = 1.0 - pow(b1, (double)t), c2 = 1.0 - pow(b2, (double)t);
    for (int64_t i = 0; i < count; i++) {
        m[i] = b1 * m[i] + (1.0 - b1) * g[i];
        v[i] = b2 * v[i] + (1.0 - b2) * g[i] * g[i];
        w[i] = w[i] - lr * (m[i] / c1) / (sqrt(v[i] / c2) + eps);
    }
    return 0;
}
