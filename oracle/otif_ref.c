/*
 * otif_ref.c — CPU ORACLE for the OTIF proxy + windowing hot path.
 *
 * TEST INFRASTRUCTURE ONLY (see otif_ref.h).  Plain C99, fp64, no blocking, no
 * fusion, no reordering beyond what the paper's procedure states, so that a
 * reader can check it against PAPER.md by eye.  Every function cites the
 * passage it follows ("P:L<n>" = line n of PAPER.md) and the DESIGN.md reading
 * (R<n>) it takes where the paper is silent.
 *
 * Parity status: resize, conv, threshold, components, grouping
 * invariants and pack are pinned by tests/test_oracle_*.py; the exact greedy
 * output beyond those pins is "parity unpinned" (the paper's worked example,
 * Fig. 3, is lost in PAPER.md).
 */
#include "otif_ref.h"

#include <math.h>
#include <stdlib.h>
#include <string.h>

/* ------------------------------------------------------------------------- */
/* bf16 rounding (reading R4): nearest bf16 value, ties to even.  bf16 has an
 * 8-bit significand and fp32's exponent range (min normal 2^-126).           */
double otif_ref_round_bf16(double x) {
    if (x == 0.0 || !isfinite(x)) return x;
    int e;
    double m = frexp(x, &e);        /* x = m * 2^e, 0.5 <= |m| < 1 */
    if (e < -125) {                 /* below bf16's normal range: fixed quantum 2^-133 */
        return ldexp(nearbyint(ldexp(x, 133)), -133);
    }
    /* 8 significant bits: quantum 2^(e-8); nearbyint() rounds half to even */
    return ldexp(nearbyint(ldexp(m, 8)), e - 8);
}

/* ------------------------------------------------------------------------- */
/* Stage 1 — resize.  P:L254 ("frames are decoded at the object detector
 * resolution"), P:L127 (the proxy "inputs video at a lower resolution").
 * Reading R13: bilinear with half-pixel centres, no antialias, round half up.
 * Source coordinate of output index y: sy = ((2y+1)·Hs − Hd) / (2·Hd), clamped
 * at 0; y0 = floor(sy), y1 = min(y0+1, Hs−1), ly = sy − y0 (same for x).      */
int otif_ref_resize(const uint8_t *src, int32_t n, int32_t sh, int32_t sw,
                    uint8_t *dst, int32_t dh, int32_t dw) {
    if (n < 0 || sh <= 0 || sw <= 0 || dh <= 0 || dw <= 0) return -1;
    for (int32_t f = 0; f < n; f++) {
        const uint8_t *s = src + (size_t)f * sh * sw * 3;
        uint8_t *d = dst + (size_t)f * dh * dw * 3;
        for (int32_t y = 0; y < dh; y++) {
            double sy = (double)((int64_t)(2 * y + 1) * sh - dh) / (double)(2 * (int64_t)dh);
            if (sy < 0.0) sy = 0.0;
            int32_t y0 = (int32_t)floor(sy);
            if (y0 > sh - 1) y0 = sh - 1;
            int32_t y1 = y0 + 1 < sh ? y0 + 1 : sh - 1;
            double ly = sy - y0;
            for (int32_t x = 0; x < dw; x++) {
                double sx = (double)((int64_t)(2 * x + 1) * sw - dw) / (double)(2 * (int64_t)dw);
                if (sx < 0.0) sx = 0.0;
                int32_t x0 = (int32_t)floor(sx);
                if (x0 > sw - 1) x0 = sw - 1;
                int32_t x1 = x0 + 1 < sw ? x0 + 1 : sw - 1;
                double lx = sx - x0;
                for (int c = 0; c < 3; c++) {
                    double p00 = s[((size_t)y0 * sw + x0) * 3 + c];
                    double p01 = s[((size_t)y0 * sw + x1) * 3 + c];
                    double p10 = s[((size_t)y1 * sw + x0) * 3 + c];
                    double p11 = s[((size_t)y1 * sw + x1) * 3 + c];
                    double v = (1.0 - ly) * ((1.0 - lx) * p00 + lx * p01)
                             + ly * ((1.0 - lx) * p10 + lx * p11);
                    double r = floor(v + 0.5);
                    if (r < 0.0) r = 0.0;
                    if (r > 255.0) r = 255.0;
                    d[((size_t)y * dw + x) * 3 + c] = (uint8_t)r;
                }
            }
        }
    }
    return 0;
}

/* ------------------------------------------------------------------------- */
/* Stage 2 — one convolution layer of the proxy CNN ("five strided
 * convolutional layers ... two additional convolutional layers").  Reading R2:
 * k x k kernel (3 or 1), zero padding (k−1)/2, ReLU; output size ceil(in/s):
 * output row o reads input rows s·o − p + kh.  Direct fp64 sum over (kh,kw,ci). */
int otif_ref_conv(const double *in, int32_t n, int32_t h, int32_t w, int32_t cin,
                  const double *weight, const double *bias, int32_t cout, int32_t k,
                  int32_t stride, int32_t relu, int32_t round_bf16, double *out) {
    if (n < 0 || h <= 0 || w <= 0 || cin <= 0 || cout <= 0) return -1;
    if (!(k == 1 || k == 3) || !(stride == 1 || stride == 2)) return -1;
    int32_t pad = (k - 1) / 2;
    int32_t ho = (h + stride - 1) / stride, wo = (w + stride - 1) / stride;
    for (int32_t f = 0; f < n; f++) {
        for (int32_t oy = 0; oy < ho; oy++) {
            for (int32_t ox = 0; ox < wo; ox++) {
                double *o = out + (((size_t)f * ho + oy) * wo + ox) * cout;
                for (int32_t co = 0; co < cout; co++) {
                    double acc = 0.0;
                    for (int32_t kh = 0; kh < k; kh++) {
                        int32_t iy = stride * oy - pad + kh;
                        if (iy < 0 || iy >= h) continue;
                        for (int32_t kw = 0; kw < k; kw++) {
                            int32_t ix = stride * ox - pad + kw;
                            if (ix < 0 || ix >= w) continue;
                            const double *x = in + (((size_t)f * h + iy) * w + ix) * cin;
                            const double *wt = weight + (((size_t)co * k + kh) * k + kw) * cin;
                            for (int32_t ci = 0; ci < cin; ci++) acc += wt[ci] * x[ci];
                        }
                    }
                    acc += bias[co];
                    if (relu && acc < 0.0) acc = 0.0;
                    if (round_bf16) acc = otif_ref_round_bf16(acc);
                    o[co] = acc;
                }
            }
        }
    }
    return 0;
}

/* Layer table of the proxy (reading R1/R2): E1..E5 3x3, D1 3x3, D2 1x1. */
static void proxy_layers(const int32_t enc[5], int32_t dec, int32_t cin[7], int32_t cout[7], int32_t ks[7]) {
    int32_t c = 3;
    for (int i = 0; i < 5; i++) { cin[i] = c; cout[i] = enc[i]; ks[i] = 3; c = enc[i]; }
    cin[5] = c;   cout[5] = dec; ks[5] = 3;
    cin[6] = dec; cout[6] = 1;   ks[6] = 1;
}

size_t otif_ref_proxy_n_weights(const int32_t enc[5], int32_t dec) {
    int32_t cin[7], cout[7], ks[7];
    proxy_layers(enc, dec, cin, cout, ks);
    size_t total = 0;
    for (int i = 0; i < 7; i++) total += (size_t)cout[i] * ks[i] * ks[i] * cin[i] + cout[i];
    return total;
}

int otif_ref_proxy_grid(int32_t in_h, int32_t in_w, int32_t n_strided, int32_t *gh, int32_t *gw) {
    if (in_h <= 0 || in_w <= 0 || n_strided < 1 || n_strided > 5) return -1;
    int32_t h = in_h, w = in_w;
    for (int i = 0; i < n_strided; i++) { h = (h + 1) / 2; w = (w + 1) / 2; }
    *gh = h; *gw = w;
    return 0;
}

/* Whole proxy ("outputs a score at each grid cell").
 * Input normalisation x = (u − 128)/128 and the sigmoid score are readings R2;
 * quantisation points are reading R4. */
int otif_ref_proxy_score(const uint8_t *img, int32_t n, int32_t in_h, int32_t in_w,
                         int32_t n_strided, const int32_t enc[5], int32_t dec,
                         const float *weights, size_t n_weights, int32_t quant,
                         double *scores) {
    int32_t gh, gw;
    if (n < 0 || otif_ref_proxy_grid(in_h, in_w, n_strided, &gh, &gw)) return -1;
    if (n_weights != otif_ref_proxy_n_weights(enc, dec)) return -2;
    if (quant != OTIF_REF_QUANT_NONE && quant != OTIF_REF_QUANT_BF16) return -3;
    int32_t cin[7], cout[7], ks[7];
    proxy_layers(enc, dec, cin, cout, ks);

    /* input: u8 -> (u − 128)/128 (exact in bf16) */
    int32_t h = in_h, w = in_w;
    double *act = (double *)malloc(sizeof(double) * (size_t)n * h * w * 3);
    if (!act) return -4;
    for (size_t i = 0; i < (size_t)n * h * w * 3; i++) act[i] = ((double)img[i] - 128.0) / 128.0;

    size_t off = 0;
    for (int L = 0; L < 7; L++) {
        size_t nw = (size_t)cout[L] * ks[L] * ks[L] * cin[L];
        double *wt = (double *)malloc(sizeof(double) * nw);
        double *bs = (double *)malloc(sizeof(double) * cout[L]);
        for (size_t i = 0; i < nw; i++) {
            double v = (double)weights[off + i];
            wt[i] = quant == OTIF_REF_QUANT_BF16 ? otif_ref_round_bf16(v) : v;
        }
        off += nw;
        for (int32_t i = 0; i < cout[L]; i++) bs[i] = (double)weights[off + i];
        off += cout[L];

        int32_t stride = (L < 5 && L < n_strided) ? 2 : 1;
        int32_t ho = (h + stride - 1) / stride, wo = (w + stride - 1) / stride;
        double *nxt = (double *)malloc(sizeof(double) * (size_t)n * ho * wo * cout[L]);
        int32_t is_head = (L == 6);
        /* E1..E5, D1: ReLU and (quant=bf16) bf16 output; D2: raw logit z */
        otif_ref_conv(act, n, h, w, cin[L], wt, bs, cout[L], ks[L], stride,
                      !is_head, (!is_head && quant == OTIF_REF_QUANT_BF16), nxt);
        free(act); free(wt); free(bs);
        act = nxt; h = ho; w = wo;
    }
    /* score = sigmoid(z): "a classification score ... indicating the likelihood" */
    for (size_t i = 0; i < (size_t)n * gh * gw; i++) scores[i] = 1.0 / (1.0 + exp(-act[i]));
    free(act);
    return 0;
}

/* ------------------------------------------------------------------------- */
/* Stage 3 — threshold ("where the score exceeds a threshold parameter
 * B_proxy"; "positive cells where the output scores exceeded B_proxy"). */
int otif_ref_threshold(const double *scores, int64_t cells, float threshold, uint8_t *mask) {
    if (cells < 0) return -1;
    double b = (double)threshold;
    for (int64_t i = 0; i < cells; i++) mask[i] = scores[i] > b ? 1 : 0;
    return 0;
}

/* ------------------------------------------------------------------------- */
/* Connected components ("we initialize a cluster c_i for each connected
 * component of positive cells").  Reading R6: 4-connectivity by default.
 * BFS; a component is seeded at the first unlabeled positive cell of a
 * row-major scan, so component indices follow raster order of their first cell. */
int otif_ref_components(const uint8_t *mask, int32_t gh, int32_t gw, int32_t connectivity,
                        int32_t *labels) {
    if (gh <= 0 || gw <= 0 || !(connectivity == 4 || connectivity == 8)) return -1;
    int32_t cells = gh * gw;
    int32_t *queue = (int32_t *)malloc(sizeof(int32_t) * cells);
    for (int32_t i = 0; i < cells; i++) labels[i] = -1;
    static const int dy8[8] = {-1, 1, 0, 0, -1, -1, 1, 1};
    static const int dx8[8] = {0, 0, -1, 1, -1, 1, -1, 1};
    int nb = connectivity == 4 ? 4 : 8;
    int32_t ncomp = 0;
    for (int32_t s = 0; s < cells; s++) {
        if (!mask[s] || labels[s] >= 0) continue;
        int32_t head = 0, tail = 0;
        queue[tail++] = s;
        labels[s] = ncomp;
        while (head < tail) {
            int32_t cur = queue[head++];
            int32_t cy = cur / gw, cx = cur % gw;
            for (int d = 0; d < nb; d++) {
                int32_t yy = cy + dy8[d], xx = cx + dx8[d];
                if (yy < 0 || yy >= gh || xx < 0 || xx >= gw) continue;
                int32_t q = yy * gw + xx;
                if (mask[q] && labels[q] < 0) { labels[q] = ncomp; queue[tail++] = q; }
            }
        }
        ncomp++;
    }
    free(queue);
    return ncomp;
}

/* ------------------------------------------------------------------------- */
/* Stage 4 — grouping cells into windows, on half-open pixel
 * rectangles [x0,x1) x [y0,y1).                                             */
typedef struct { int32_t x0, y0, x1, y1; } rect;

/* W' = W sorted by (cost, w·h, w, h): canonical order (reading R7/R8). */
static int wsize_less(const otif_ref_wsize *a, const otif_ref_wsize *b) {
    if (a->cost != b->cost) return a->cost < b->cost;
    int64_t aa = (int64_t)a->w * a->h, ba = (int64_t)b->w * b->h;
    if (aa != ba) return aa < ba;
    if (a->w != b->w) return a->w < b->w;
    return a->h < b->h;
}

/* fit(r) = first s in W' with s.w >= r.w and s.h >= r.h: the cheapest size
 * that contains the cluster ("(r_i.w, r_i.h) ∈ W"). */
static int fit(const rect *r, const otif_ref_wsize *sizes, const int32_t *order, int32_t k) {
    int32_t rw = r->x1 - r->x0, rh = r->y1 - r->y0;
    for (int32_t t = 0; t < k; t++) {
        const otif_ref_wsize *s = &sizes[order[t]];
        if (s->w >= rw && s->h >= rh) return order[t];
    }
    return -1;
}

static rect runion(const rect *a, const rect *b) {
    rect u;
    u.x0 = a->x0 < b->x0 ? a->x0 : b->x0;
    u.y0 = a->y0 < b->y0 ? a->y0 : b->y0;
    u.x1 = a->x1 > b->x1 ? a->x1 : b->x1;
    u.y1 = a->y1 > b->y1 ? a->y1 : b->y1;
    return u;
}

static int32_t clampi(int32_t v, int32_t lo, int32_t hi) { return v < lo ? lo : (v > hi ? hi : v); }

/* place(r) (reading R9): size s = fit(r); window centred on the cluster bbox
 * with floor on the half-difference, then clamped inside the frame. */
static void place(const rect *r, const otif_ref_wsize *s, int32_t fw, int32_t fh, int32_t *x, int32_t *y) {
    int32_t rw = r->x1 - r->x0, rh = r->y1 - r->y0;
    *x = clampi(r->x0 - (s->w - rw) / 2, 0, fw - s->w);
    *y = clampi(r->y0 - (s->h - rh) / 2, 0, fh - s->h);
}

int otif_ref_group_frame(const uint8_t *mask, int32_t gh, int32_t gw, int32_t cell,
                         int32_t frame_w, int32_t frame_h, int32_t connectivity,
                         const otif_ref_wsize *sizes, int32_t k, int32_t frame_index,
                         otif_ref_window *out, int32_t cap) {
    if (gh <= 0 || gw <= 0 || cell <= 0 || frame_w <= 0 || frame_h <= 0 || k <= 0) return -1;
    if (gh != (frame_h + cell - 1) / cell || gw != (frame_w + cell - 1) / cell) return -1;
    int have_full = 0;
    for (int32_t t = 0; t < k; t++) {
        if (sizes[t].w <= 0 || sizes[t].h <= 0 || sizes[t].w > frame_w || sizes[t].h > frame_h) return -1;
        if (sizes[t].w == frame_w && sizes[t].h == frame_h) have_full = 1;
    }
    if (!have_full) return -1; /* "we always include this maximum window size" */

    /* W' order (insertion sort, k is tiny) */
    int32_t *order = (int32_t *)malloc(sizeof(int32_t) * k);
    for (int32_t t = 0; t < k; t++) order[t] = t;
    for (int32_t a = 1; a < k; a++)
        for (int32_t b = a; b > 0 && wsize_less(&sizes[order[b]], &sizes[order[b - 1]]); b--) {
            int32_t tmp = order[b]; order[b] = order[b - 1]; order[b - 1] = tmp;
        }

    /* connected components, then one cluster per component, bbox in pixels
     * (cells are c x c detector pixels, the edge cell clipped: reading R14) */
    int32_t cells = gh * gw;
    int32_t *labels = (int32_t *)malloc(sizeof(int32_t) * cells);
    int32_t n = otif_ref_components(mask, gh, gw, connectivity, labels);
    if (n <= 0) { free(labels); free(order); return n; }
    rect *cl = (rect *)malloc(sizeof(rect) * n);
    int *alive = (int *)malloc(sizeof(int) * n);
    for (int32_t i = 0; i < n; i++) { cl[i].x0 = cl[i].y0 = 1 << 30; cl[i].x1 = cl[i].y1 = -1; alive[i] = 1; }
    for (int32_t q = 0; q < cells; q++) {
        int32_t l = labels[q];
        if (l < 0) continue;
        int32_t cy = q / gw, cx = q % gw;
        int32_t x0 = cx * cell, y0 = cy * cell;
        int32_t x1 = (cx + 1) * cell < frame_w ? (cx + 1) * cell : frame_w;
        int32_t y1 = (cy + 1) * cell < frame_h ? (cy + 1) * cell : frame_h;
        if (x0 < cl[l].x0) cl[l].x0 = x0;
        if (y0 < cl[l].y0) cl[l].y0 = y0;
        if (x1 > cl[l].x1) cl[l].x1 = x1;
        if (y1 > cl[l].y1) cl[l].y1 = y1;
    }

    for (;;) {
        /* Phase A: "repeatedly check whether two clusters can be combined
         * to form a merged cluster that would be faster to process ... (i.e.,
         * whether merging would decrease est(R))".  Reading R7: take the pair with
         * the largest decrease, ties to the lexicographically smallest (i, j) in
         * current cluster order; stop when no merge strictly decreases est. */
        for (;;) {
            int64_t best = 0;
            int32_t bi = -1, bj = -1;
            for (int32_t i = 0; i < n; i++) {
                if (!alive[i]) continue;
                int64_t ci = sizes[fit(&cl[i], sizes, order, k)].cost;
                for (int32_t j = i + 1; j < n; j++) {
                    if (!alive[j]) continue;
                    int64_t cj = sizes[fit(&cl[j], sizes, order, k)].cost;
                    rect u = runion(&cl[i], &cl[j]);
                    int64_t cu = sizes[fit(&u, sizes, order, k)].cost;
                    int64_t g = ci + cj - cu;
                    if (g > best) { best = g; bi = i; bj = j; }
                }
            }
            if (bi < 0) break; /* "Once merging offers no further improvement" */
            cl[bi] = runion(&cl[bi], &cl[bj]);
            alive[bj] = 0;
        }
        /* Phase B (reading R10): windows must be disjoint; merge the
         * lexicographically first pair whose placed windows overlap, then
         * return to phase A.  Terminates: every merge removes a cluster. */
        int32_t oi = -1, oj = -1;
        for (int32_t i = 0; i < n && oi < 0; i++) {
            if (!alive[i]) continue;
            int32_t si = fit(&cl[i], sizes, order, k), xi, yi;
            place(&cl[i], &sizes[si], frame_w, frame_h, &xi, &yi);
            for (int32_t j = i + 1; j < n; j++) {
                if (!alive[j]) continue;
                int32_t sj = fit(&cl[j], sizes, order, k), xj, yj;
                place(&cl[j], &sizes[sj], frame_w, frame_h, &xj, &yj);
                int ox = xi < xj + sizes[sj].w && xj < xi + sizes[si].w;
                int oy = yi < yj + sizes[sj].h && yj < yi + sizes[si].h;
                if (ox && oy) { oi = i; oj = j; break; }
            }
        }
        if (oi < 0) break;
        cl[oi] = runion(&cl[oi], &cl[oj]);
        alive[oj] = 0;
    }

    /* R = one rectangle per final cluster */
    int32_t m = 0;
    int64_t est = 0;
    otif_ref_window *R = (otif_ref_window *)malloc(sizeof(otif_ref_window) * n);
    for (int32_t i = 0; i < n; i++) {
        if (!alive[i]) continue;
        int32_t s = fit(&cl[i], sizes, order, k), x, y;
        place(&cl[i], &sizes[s], frame_w, frame_h, &x, &y);
        R[m].frame = frame_index; R[m].x = x; R[m].y = y;
        R[m].w = sizes[s].w; R[m].h = sizes[s].h; R[m].size_idx = s;
        est += sizes[s].cost;
        m++;
    }
    /* "falling back to detecting objects in the entire frame when doing
     * so would be faster" — strict (reading R11). */
    rect full = {0, 0, frame_w, frame_h};
    int32_t sfull = fit(&full, sizes, order, k);
    if (est > sizes[sfull].cost) {
        m = 1;
        R[0].frame = frame_index; R[0].x = 0; R[0].y = 0;
        R[0].w = frame_w; R[0].h = frame_h; R[0].size_idx = sfull;
    }
    /* emit sorted by (y, x) (reading R15) */
    for (int32_t a = 1; a < m; a++)
        for (int32_t b = a; b > 0 && (R[b].y < R[b - 1].y || (R[b].y == R[b - 1].y && R[b].x < R[b - 1].x)); b--) {
            otif_ref_window t = R[b]; R[b] = R[b - 1]; R[b - 1] = t;
        }
    for (int32_t i = 0; i < m && i < cap; i++) out[i] = R[i];
    free(R); free(alive); free(cl); free(labels); free(order);
    return m;
}

int otif_ref_select_windows(const uint8_t *mask, int32_t n, int32_t gh, int32_t gw,
                            int32_t cell, int32_t frame_w, int32_t frame_h, int32_t connectivity,
                            const otif_ref_wsize *sizes, int32_t k,
                            otif_ref_window *windows, int32_t capacity,
                            int32_t *frame_count, int32_t *frame_offset, int32_t *total) {
    if (n < 0 || capacity < 0) return -1;
    int32_t cells = gh * gw;
    otif_ref_window *tmp = (otif_ref_window *)malloc(sizeof(otif_ref_window) * (cells + 1));
    int64_t run = 0;
    for (int32_t f = 0; f < n; f++) {
        int r = otif_ref_group_frame(mask + (size_t)f * cells, gh, gw, cell, frame_w, frame_h,
                                     connectivity, sizes, k, f, tmp, cells + 1);
        if (r < 0) { free(tmp); return r; }
        frame_count[f] = r;
        frame_offset[f] = (int32_t)run;
        for (int32_t i = 0; i < r; i++)
            if (run + i < capacity) windows[run + i] = tmp[i];
        run += r;
    }
    *total = (int32_t)run;
    free(tmp);
    return 0;
}

/* ------------------------------------------------------------------------- */
/* Stage 5 — crop/pack ("initializes the detector on the GPU to execute
 * at each of those sizes"; "batching many equal-dimension inputs together"). */
int otif_ref_pack_windows(const uint8_t *src, int32_t n, int32_t sh, int32_t sw,
                          int32_t det_h, int32_t det_w,
                          const otif_ref_window *windows, int32_t total,
                          const otif_ref_wsize *sizes, int32_t k,
                          uint8_t *const *batches, const int32_t *batch_cap,
                          int32_t *slot, int32_t *size_count) {
    if (n < 0 || total < 0 || k <= 0) return -1;
    const uint8_t *det = src;
    uint8_t *owned = NULL;
    if (det_h != sh || det_w != sw) {
        owned = (uint8_t *)malloc((size_t)n * det_h * det_w * 3);
        otif_ref_resize(src, n, sh, sw, owned, det_h, det_w);
        det = owned;
    }
    for (int32_t s = 0; s < k; s++) size_count[s] = 0;
    for (int32_t g = 0; g < total; g++) {
        const otif_ref_window *r = &windows[g];
        int32_t s = r->size_idx;
        int32_t sl = size_count[s]++;
        slot[g] = sl;
        if (sl >= batch_cap[s]) continue;
        uint8_t *dst = batches[s] + (size_t)sl * sizes[s].h * sizes[s].w * 3;
        const uint8_t *fr = det + (size_t)r->frame * det_h * det_w * 3;
        for (int32_t yy = 0; yy < r->h; yy++)
            memcpy(dst + (size_t)yy * r->w * 3,
                   fr + ((size_t)(r->y + yy) * det_w + r->x) * 3, (size_t)r->w * 3);
    }
    free(owned);
    return 0;
}

/* ------------------------------------------------------------------------- */
/* est(R_t) = Σ_{r in R_t} T_{r.w, r.h} of the windows stage 4 emits. */
int64_t otif_ref_frame_est(const uint8_t *mask, int32_t gh, int32_t gw, int32_t cell, int32_t frame_w,
                           int32_t frame_h, int32_t connectivity, const otif_ref_wsize *sizes, int32_t k) {
    int32_t cap = gh * gw + 1;
    otif_ref_window *R = (otif_ref_window *)malloc(sizeof(otif_ref_window) * cap);
    int m = otif_ref_group_frame(mask, gh, gw, cell, frame_w, frame_h, connectivity, sizes, k, 0, R, cap);
    int64_t est = 0;
    for (int i = 0; i < m; i++) est += sizes[R[i].size_idx].cost;
    free(R);
    return m < 0 ? -1 : est;
}

/* NEXT-1 — P:L155: "we first initialize W to only contain the size corresponding to the
 * entire video frame ... We then repeatedly greedily add the window size to W that
 * provides the greatest decrease to Σ_t est(R(I_t; W)), until |W| = k." */
int otif_ref_choose_window_sizes(const uint8_t *masks, int32_t n, int32_t gh, int32_t gw, int32_t cell,
                                 int32_t frame_w, int32_t frame_h, int32_t connectivity,
                                 const otif_ref_wsize *candidates, int32_t m, int64_t full_cost, int32_t k,
                                 int32_t *chosen_idx, int64_t *est) {
    if (n < 0 || m < 0 || k < 1) return -1;
    otif_ref_wsize *W = (otif_ref_wsize *)malloc(sizeof(otif_ref_wsize) * (k + 1));
    int32_t *used = (int32_t *)calloc(m > 0 ? m : 1, sizeof(int32_t));
    W[0].w = frame_w; W[0].h = frame_h; W[0].cost = full_cost;
    int32_t nw = 1;
    int64_t cur = 0;
    for (int32_t f = 0; f < n; f++)
        cur += otif_ref_frame_est(masks + (size_t)f * gh * gw, gh, gw, cell, frame_w, frame_h, connectivity, W, nw);
    chosen_idx[0] = -1;
    est[0] = cur;
    while (nw < k) {
        int32_t best = -1;
        int64_t best_sum = cur;
        for (int32_t c = 0; c < m; c++) {
            if (used[c]) continue;
            W[nw] = candidates[c];
            int64_t sum = 0;
            for (int32_t f = 0; f < n; f++)
                sum += otif_ref_frame_est(masks + (size_t)f * gh * gw, gh, gw, cell, frame_w, frame_h, connectivity,
                                          W, nw + 1);
            if (sum < best_sum) { best_sum = sum; best = c; }  /* greatest decrease; ties: earliest */
        }
        if (best < 0) break;  /* no candidate decreases the sum (reading R19) */
        used[best] = 1;
        W[nw] = candidates[best];
        chosen_idx[nw] = best;
        est[nw] = best_sum;
        cur = best_sum;
        nw++;
    }
    free(W);
    free(used);
    return nw;
}

/* NEXT-2 — P:L232: "The recall is the fraction of detections computed by θ_best that are
 * covered by rectangles in R_ij"; reading R18: contained in one window of its frame. */
int64_t otif_ref_covered(const int32_t *boxes, int64_t nb, const otif_ref_window *windows, int32_t total) {
    int64_t covered = 0;
    for (int64_t i = 0; i < nb; i++) {
        const int32_t *b = boxes + i * 5;
        for (int32_t g = 0; g < total; g++) {
            const otif_ref_window *r = &windows[g];
            if (r->frame != b[0]) continue;
            if (r->x <= b[1] && b[3] <= r->x + r->w && r->y <= b[2] && b[4] <= r->y + r->h) { covered++; break; }
        }
    }
    return covered;
}
