/*
 * otif_ref.h — CPU ORACLE for the OTIF proxy + windowing hot path.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs may load this library.  The product path
 * (paper_conf_sigmod_bastanim22_b200/) never links, imports or calls it, and this
 * code shares nothing with the CUDA path (no headers, helpers or tables).
 *
 * Plain, slow, single-threaded C99 in fp64, following PAPER.md (OTIF, Bastani &
 * Madden, SIGMOD'22) step by step; readings where the paper is silent are the
 * ones listed in DESIGN.md §3 (SURVEY.md §8(c) R1–R17).  Citations "P:L<n>" are
 * lines of /root/reference/PAPER.md.
 *
 * All pointers are HOST pointers.  Layouts: images u8 NHWC RGB (C = 3),
 * activations fp64 NHWC, weights fp32 W[Cout][kh][kw][Cin] followed by b[Cout].
 * Every function returns 0 on success and a negative value on bad arguments.
 */
#ifndef OTIF_REF_H
#define OTIF_REF_H
#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* quantisation modes of the proxy (reading R4) */
#define OTIF_REF_QUANT_NONE 0 /* no rounding anywhere: pure fp64 */
#define OTIF_REF_QUANT_BF16 1 /* weights and every inter-layer activation rounded to bf16 (RNE) */

typedef struct { int32_t w, h; int64_t cost; } otif_ref_wsize;                /* (w,h) in W with T_{w,h} */
typedef struct { int32_t frame, x, y, w, h, size_idx; } otif_ref_window;      /* r = (x,y,w,h) */

/* Round an fp64 value to the nearest bf16 value, ties to even (reading R4). */
double otif_ref_round_bf16(double x);

/* Stage 1: bilinear resize, half-pixel centres, no antialias,
 * round half up, u8 NHWC, C = 3.  src [n,sh,sw,3] -> dst [n,dh,dw,3]. */
int otif_ref_resize(const uint8_t *src, int32_t n, int32_t sh, int32_t sw,
                    uint8_t *dst, int32_t dh, int32_t dw);

/* Stage 2, one layer: 3x3 conv (or 1x1 when k == 1), zero pad (k-1)/2,
 * stride s in {1,2}, + bias, optional ReLU, optional bf16 rounding of the output.
 * in [n,h,w,cin] fp64 -> out [n,ceil(h/s),ceil(w/s),cout] fp64.
 * w/b are used exactly as given (caller pre-rounds weights for quant=bf16). */
int otif_ref_conv(const double *in, int32_t n, int32_t h, int32_t w, int32_t cin,
                  const double *weight, const double *bias, int32_t cout, int32_t k,
                  int32_t stride, int32_t relu, int32_t round_bf16, double *out);

/* Stage 2, whole proxy.  Encoder widths enc[5], decoder
 * width dec; the first n_strided encoder layers have stride 2 (reading R1).
 * weights: fp32 blob E1..E5, D1, D2.  img [n,in_h,in_w,3] u8 -> scores [n,gh,gw]
 * fp64 with gh = ceil(in_h / 2^n_strided).  quant: OTIF_REF_QUANT_*. */
size_t otif_ref_proxy_n_weights(const int32_t enc[5], int32_t dec);
int otif_ref_proxy_grid(int32_t in_h, int32_t in_w, int32_t n_strided, int32_t *gh, int32_t *gw);
int otif_ref_proxy_score(const uint8_t *img, int32_t n, int32_t in_h, int32_t in_w,
                         int32_t n_strided, const int32_t enc[5], int32_t dec,
                         const float *weights, size_t n_weights, int32_t quant,
                         double *scores);

/* Stage 3 ("exceeds"): mask = score > B, strict, compared in fp64. */
int otif_ref_threshold(const double *scores, int64_t cells, float threshold, uint8_t *mask);

/* Connected components: BFS seeded in row-major order; labels[gh*gw]
 * = component index in seed order, -1 for negative cells.  Returns the count. */
int otif_ref_components(const uint8_t *mask, int32_t gh, int32_t gw, int32_t connectivity,
                        int32_t *labels);

/* Stage 4 for one frame: windows covering the positive cells,
 * greedy agglomerative merge, disjointness pass, full-frame fallback
 * (P:L133).  Writes at most cap windows sorted by (y, x); returns the count
 * (which may exceed cap) or a negative error. */
int otif_ref_group_frame(const uint8_t *mask, int32_t gh, int32_t gw, int32_t cell,
                         int32_t frame_w, int32_t frame_h, int32_t connectivity,
                         const otif_ref_wsize *sizes, int32_t k, int32_t frame_index,
                         otif_ref_window *out, int32_t cap);

/* Stage 4 over a batch: compacted windows in (frame, y, x) order, counts,
 * exclusive offsets, total.  Returns 0 (total is exact even if > capacity). */
int otif_ref_select_windows(const uint8_t *mask, int32_t n, int32_t gh, int32_t gw,
                            int32_t cell, int32_t frame_w, int32_t frame_h, int32_t connectivity,
                            const otif_ref_wsize *sizes, int32_t k,
                            otif_ref_window *windows, int32_t capacity,
                            int32_t *frame_count, int32_t *frame_offset, int32_t *total);

/* Stage 5: det = resize(src -> det_h x det_w) (a copy when
 * equal); for windows in order, slot = running count of its size_idx;
 * batches[s][slot] = det[frame][y:y+h, x:x+w, :].  Entries with slot >=
 * batch_cap[s] are dropped; size_count[s] is exact. */
int otif_ref_pack_windows(const uint8_t *src, int32_t n, int32_t sh, int32_t sw,
                          int32_t det_h, int32_t det_w,
                          const otif_ref_window *windows, int32_t total,
                          const otif_ref_wsize *sizes, int32_t k,
                          uint8_t *const *batches, const int32_t *batch_cap,
                          int32_t *slot, int32_t *size_count);

/* est(R_t) of one frame's windows: Σ T over the windows stage 4 emits. */
int64_t otif_ref_frame_est(const uint8_t *mask, int32_t gh, int32_t gw, int32_t cell, int32_t frame_w,
                           int32_t frame_h, int32_t connectivity, const otif_ref_wsize *sizes, int32_t k);

/* NEXT-1: choose the fixed window-size set.  "we first initialize W to only
 * contain the size corresponding to the entire video frame ... We then repeatedly greedily
 * add the window size to W that provides the greatest decrease to Σ_t est(R(I_t; W)),
 * until |W| = k", over perfect-proxy masks.  candidates: m sizes (the full frame
 * excluded); ties go to the earliest candidate; stops early when no candidate decreases
 * the sum (reading R19).  chosen_idx[k]: candidate index of each added size (-1 = the
 * full frame, always chosen_idx[0]); est[k]: Σ_t est after each addition.  Returns the
 * number of sizes chosen (<= k). */
int otif_ref_choose_window_sizes(const uint8_t *masks, int32_t n, int32_t gh, int32_t gw, int32_t cell,
                                 int32_t frame_w, int32_t frame_h, int32_t connectivity,
                                 const otif_ref_wsize *candidates, int32_t m, int64_t full_cost, int32_t k,
                                 int32_t *chosen_idx, int64_t *est);

/* NEXT-2: recall = fraction of detections "covered by rectangles" — a
 * detection [x0,x1) x [y0,y1) (clipped to the frame) counts as covered when it lies
 * inside one window of its frame (reading R18).  boxes: int32 [nb][5] = (frame, x0, y0,
 * x1, y1); windows/total as from otif_ref_select_windows.  Returns the covered count. */
int64_t otif_ref_covered(const int32_t *boxes, int64_t nb, const otif_ref_window *windows, int32_t total);

/* ------------------------------------------------------------------------- */
/* NEXT-4: track refinement, otif_ref_tracks.c.  A track is a sequence of
 * detection centres (x, y) (reading R20): pts float32 [total][2], offsets int64 [n+1].
 * These functions take the integer decisions (neighbour, core, nearest) in fp32, the
 * kernel's precision (R21–R25), and compute resampled points and centres in
 * fp64 with a fixed operation order, so that the GPU can match them bit for bit.      */

/* P:L196 "we compute N points evenly spaced along each track": arc-length resampling
 * (reading R21).  out float32 [n][npts][2]. */
int otif_ref_track_resample(const float *pts, const int64_t *offsets, int64_t n, int32_t npts, float *out);

/* P:L196 d(s1, s2) = (1/N) Σ_i eucl(P(s1)[i], P(s2)[i]), fp32 (reading R22). */
float otif_ref_track_distance(const float *a, const float *b, int32_t npts);

/* P:L198 DBSCAN over resampled tracks P [n][npts][2] (reading R23): neighbours d <= eps
 * (a track is its own neighbour), core iff |neighbours| >= min_pts, clusters = connected
 * components of core tracks numbered by their smallest index, a border track joins the
 * smallest-numbered cluster among its core neighbours, noise = -1.  labels int32 [n];
 * core u8 [n] (may be NULL).  Returns the number of clusters. */
int32_t otif_ref_dbscan(const float *P, int64_t n, int32_t npts, float eps, int32_t min_pts, int32_t *labels,
                        uint8_t *core);

/* P:L198 "the center of a cluster ... p_i is the average of points in {P(s)[i] | s ∈ c}":
 * fp64 sum over members in index order, divided by the count, rounded to fp32.
 * centers float32 [nc][npts][2], sizes int32 [nc]. */
int otif_ref_track_centers(const float *P, const int32_t *labels, int64_t n, int32_t npts, int32_t nc,
                           float *centers, int32_t *sizes);

/* P:L200 refinement of query tracks (raw pts/offsets, m tracks): candidates = cluster
 * centres passing within rho of the first AND the last detection (rho <= 0: all centres;
 * reading R24); keep the k closest by (d, cluster index); start/end = per-coordinate lower
 * weighted median of the kept centres' first/last points, weights = cluster sizes (reading
 * R25).  out float32 [m][4] = (start x, start y, end x, end y); a track with no candidate
 * keeps its own first/last detection.  used int32 [m] = number of clusters kept. */
int otif_ref_track_refine(const float *pts, const int64_t *offsets, int64_t m, int32_t npts, const float *centers,
                          const int32_t *sizes, int32_t nc, int32_t k, float rho, float *out, int32_t *used);

/* ------------------------------------------------------------------------- */
/* NEXT-3: proxy training labels and training, otif_ref_train.c, fp64. */

/* label 1 at a cell some detection intersects.  boxes int32 [nb][5] = (frame,
 * x0, y0, x1, y1), half-open pixels; labels u8 [n][gh][gw]. */
int otif_ref_cell_labels(const int32_t *boxes, int64_t nb, int32_t n, int32_t gh, int32_t gw, int32_t cell,
                         int32_t frame_w, int32_t frame_h, uint8_t *labels);

/* Backward of one convolution (pad (k−1)/2, stride 1 or 2) given dy = ∂L/∂(conv output):
 * dx [n,h,w,cin] (may be NULL), dW [cout][k][k][cin], db [cout] — overwritten. */
int otif_ref_conv_backward(const double *x, int32_t n, int32_t h, int32_t w, int32_t cin, const double *weight,
                           int32_t cout, int32_t k, int32_t stride, const double *dy, double *dx, double *dW,
                           double *db);

/* One batch: forward (quant none), mean BCE-with-logits loss vs labels (reading R26),
 * gradient of every weight and bias (fp64 blob in the proxy weight layout). */
int otif_ref_proxy_grad(const uint8_t *img, int32_t n, int32_t in_h, int32_t in_w, int32_t n_strided,
                        const int32_t enc[5], int32_t dec, const double *weights, const uint8_t *labels,
                        double *loss, double *grad);

/* Adam step t >= 1 (reading R27), in place on w, m, v. */
int otif_ref_adam(double *w, double *m, double *v, const double *g, int64_t count, int32_t t, double lr, double b1,
                  double b2, double eps);

#ifdef __cplusplus
}
#endif
#endif
