/*
 * otif.h — C ABI of the B200-native (sm_100a) OTIF proxy + windowing hot path.
 *
 * OTIF (Bastani & Madden, SIGMOD'22) runs, on every sampled frame, a segmentation
 * proxy that scores each grid cell, thresholds the scores, groups the positive
 * cells into rectangular windows of a few fixed sizes, and runs the detector on
 * those windows in equal-size batches.  This library is that per-frame path.
 * Citations "P:L<n>" are lines of the paper text; readings R<n> are
 * listed in DESIGN.md §3.
 *
 * Conventions (all entry points):
 *  - Pointers are CUDA DEVICE pointers unless marked [host].  All buffers are
 *    allocated and owned by the caller; the library never allocates device memory
 *    except in otif_proxy_create (packed weights) and otif_pipeline_create.
 *  - Every call only enqueues work on `stream` and returns; it never synchronises.
 *    The return value reports synchronous argument validation and launch errors;
 *    asynchronous faults surface at the caller's next synchronisation.
 *  - Images are u8 NHWC RGB (C = 3), rows densely packed (row stride 3*W bytes).
 *  - No exception crosses the ABI and there is no CPU fallback: every stage runs in
 *    this library's sm_100a kernels.  OTIF_EUNSUPPORTED is returned on a device
 *    that is not sm_100 or for shapes the kernels do not cover.
 */
#ifndef OTIF_H
#define OTIF_H

#include <stddef.h>
#include <stdint.h>
#include <cuda_runtime_api.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
    OTIF_OK = 0,
    OTIF_EINVAL = 1,        /* bad argument (shape, NULL pointer, inconsistent sizes) */
    OTIF_ENOMEM = 2,        /* allocation in *_create failed, or workspace too small */
    OTIF_ECUDA = 3,         /* a CUDA runtime call or kernel launch failed */
    OTIF_EUNSUPPORTED = 4   /* not an sm_100 device, or a shape beyond the kernels' limits */
} otif_status;

const char *otif_status_str(otif_status s);
/* Thread-local human-readable detail for the last non-OK status of this thread. */
const char *otif_last_error(void);
/* Library version string, e.g. "otif-b200 0.1 sm_100a". */
const char *otif_version(void);

/* An element of the window-size set W with its detector time T_{w,h}.
 * Costs are integers so that merge decisions and ties are exact (reading R8);
 * the default is the window area w*h. */
typedef struct { int32_t w, h; int64_t cost; } otif_wsize;

/* A window r = (x, y, w, h) in detector pixels, half-open, (w, h) = sizes[size_idx]
 * ("each r_i is a 4-tuple (r_i.x, r_i.y, r_i.w, r_i.h) ... (r_i.w, r_i.h) ∈ W"). */
typedef struct { int32_t frame, x, y, w, h, size_idx; } otif_window;

/* ---------------------------------------------------------------------------
 * Stage 1 — resize (frames are decoded at the detector resolution and the
 * proxy "inputs video at a lower resolution").  Bilinear with half-pixel
 * centres, no antialias, fp32 blend, round half up (reading R13).
 *   src [n, src_h, src_w, 3] u8  ->  dst [n, dst_h, dst_w, 3] u8.
 * Any positive sizes (down- or up-scaling).  src and dst must not overlap.
 * Errors: OTIF_EINVAL for non-positive sizes or NULL pointers. */
otif_status otif_resize(const uint8_t *src, int32_t n, int32_t src_h, int32_t src_w,
                        uint8_t *dst, int32_t dst_h, int32_t dst_w, cudaStream_t stream);

/* ---------------------------------------------------------------------------
 * Stage 2 — segmentation proxy CNN ("a five-layer encoder followed
 * by a two-layer decoder ... a classification score at each ... cell").
 * Shape (readings R1, R2): E1..E5 3x3 pad 1 + ReLU with widths enc[0..4]; the first
 * n_strided (= log2 S, 1..5) encoder layers have stride 2; D1 3x3 pad 1 + ReLU
 * (width dec); D2 1x1 -> 1 logit; score = sigmoid(logit).  Input (u - 128)/128.
 * Precision (reading R4): bf16 weights and activations (RNE after bias + ReLU),
 * fp32 accumulation on the tensor cores, fp32 logit and score.
 * Supported widths: enc[0] == 32; enc[1..4] and dec in {64, 128, 256}; dec <= 256. */
typedef struct {
    int32_t in_h, in_w;     /* proxy input resolution */
    int32_t n_strided;      /* log2 of the output stride S, 1..5 */
    int32_t enc[5];         /* encoder widths */
    int32_t dec;            /* decoder width (D1) */
} otif_proxy_desc;

typedef struct otif_proxy otif_proxy;

/* weights: [host] fp32 blob, layers E1..E5, D1, D2 in order; per layer
 * W[Cout][kh][kw][Cin] then b[Cout] (n_weights must match the descriptor).
 * The handle owns the weights repacked (bf16, tap-major K blocks) in device memory;
 * it is immutable after creation and may be shared by several streams.
 * Uses the current CUDA device. */
otif_status otif_proxy_create(const otif_proxy_desc *d, const float *weights, size_t n_weights,
                              otif_proxy **out);
void otif_proxy_destroy(otif_proxy *p);
/* Output grid (gh, gw) = (ceil(in_h / S), ceil(in_w / S)). */
otif_status otif_proxy_grid(const otif_proxy *p, int32_t *gh, int32_t *gw);
/* Device workspace needed for a batch of n frames (activations between layers). */
size_t otif_proxy_workspace_bytes(const otif_proxy *p, int32_t n);
/* img [n, in_h, in_w, 3] u8 -> scores [n, gh, gw] fp32.
 * workspace: >= otif_proxy_workspace_bytes(p, n) bytes, 256-B aligned.  It is
 * initialised by the library on first use (a header tag records the layout) and
 * must not be written by the caller between calls; a caller that reuses the memory
 * for something else must zero its first 256 bytes before handing it back. */
otif_status otif_proxy_score(const otif_proxy *p, const uint8_t *img, int32_t n, float *scores,
                             void *workspace, size_t ws_bytes, cudaStream_t stream);

/* ---------------------------------------------------------------------------
 * Stages 3 + 4 — threshold and window selection ("After thresholding the
 * scores by B_proxy, we derive a binary grid ... of positive cells"; P:L149–151:
 * windows R_t with sizes in W covering every positive cell, found by greedy
 * agglomerative merging of connected components while est(R) = Σ T decreases;
 * fall back to the full frame when that is faster).  Exact algorithm:
 * DESIGN.md §3 (readings R6–R11, R14, R15).  Integer arithmetic throughout.
 *   exactly one of scores [n, gh, gw] fp32 / mask_in [n, gh, gw] u8 (0/1) is non-NULL;
 *   mask_in is the "perfect proxy" mode of P:L153.  mask = scores > threshold.
 *   sizes: [host] W, k entries (1 <= k <= 8); must contain (frame_w, frame_h)
 *    and no size larger than the frame.
 * Outputs: mask_out [n, gh, gw] u8 (optional, may be NULL); windows [capacity]
 * compacted across the batch in (frame, y, x) order; frame_count[n], frame_offset[n]
 * (exclusive prefix), total[1].  total and counts are exact even when windows beyond
 * `capacity` are dropped; capacity = n*ceil(gh*gw/2) can never overflow.
 * est_sum [1] int64 (device, optional, may be NULL): set to Σ_t est(R_t) over the n
 * frames, est(R) = Σ_{r in R} T_{r.w, r.h} (the runtime estimate the tuner
 * sums) — computed with the grouping, no second pass.
 * Limits: gh*gw <= 8192.  workspace: >= otif_select_workspace_bytes(n, gh, gw). */
typedef struct { int32_t frame_w, frame_h, cell, connectivity; /* 4 or 8 */ } otif_grid_desc;
size_t otif_select_workspace_bytes(int32_t n, int32_t gh, int32_t gw);
otif_status otif_select_windows(const float *scores, const uint8_t *mask_in, float threshold,
                                int32_t n, int32_t gh, int32_t gw, const otif_grid_desc *g,
                                const otif_wsize *sizes, int32_t k,
                                uint8_t *mask_out, otif_window *windows, int32_t capacity,
                                int32_t *frame_count, int32_t *frame_offset, int32_t *total,
                                void *workspace, size_t ws_bytes, cudaStream_t stream, int64_t *est_sum);

/* ---------------------------------------------------------------------------
 * Stage 5 — crop / resample / pack (the detector is initialised "at each of
 * those sizes" and "high detection performance on GPUs relies heavily on batching
 * many equal-dimension inputs together").
 *   det = resize(src -> det_h x det_w) (bilinear as in stage 1; a plain copy when
 *   equal); for the windows[0 .. min(*total, capacity)) in order, slot = running
 *   count of its size_idx; batches[s][slot] = det[frame][y:y+h, x:x+w, :].
 *   batches: [host] array of k device pointers, batches[s] is [batch_cap[s], h_s, w_s, 3].
 *   batch_cap: [host] k capacities.  slot [capacity] int32 and size_count [k] are
 *   device outputs; size_count is exact even when entries beyond batch_cap are dropped.
 * `total` is read on the device (no host synchronisation). */
otif_status otif_pack_windows(const uint8_t *src, int32_t n, int32_t src_h, int32_t src_w,
                              int32_t det_h, int32_t det_w,
                              const otif_window *windows, const int32_t *total, int32_t capacity,
                              const otif_wsize *sizes, int32_t k,
                              uint8_t *const *batches, const int32_t *batch_cap,
                              int32_t *slot, int32_t *size_count, cudaStream_t stream);

/* ---------------------------------------------------------------------------
 * §8(f) NEXT-1 — choosing the fixed window sizes W: "we first initialize W
 * to only contain the size corresponding to the entire video frame ... We then
 * repeatedly greedily add the window size to W that provides the greatest decrease to
 * Σ_t est(R(I_t; W)), until |W| = k", assuming a perfect proxy (masks = ground-truth
 * cells).  masks [n, gh, gw] u8 (device); candidates [host] m sizes (the full
 * frame is implicit, cost full_cost); ties go to the earliest candidate; the loop stops
 * early when no candidate decreases the sum (reading R19).  Outputs [host]:
 * chosen_idx[k] (-1 = full frame at [0], candidate index after, -2 = not filled) and
 * est[k] (Σ_t est after each addition).  Synchronises `stream` once per round.
 * workspace: >= otif_choose_workspace_bytes(n, gh, gw, m). */
size_t otif_choose_workspace_bytes(int32_t n, int32_t gh, int32_t gw, int32_t m);
otif_status otif_choose_window_sizes(const uint8_t *masks, int32_t n, int32_t gh, int32_t gw,
                                     const otif_grid_desc *g, const otif_wsize *candidates, int32_t m,
                                     int64_t full_cost, int32_t k, int32_t *chosen_idx, int64_t *est,
                                     void *workspace, size_t ws_bytes, cudaStream_t stream);

/* §8(f) NEXT-2 — proxy tuning: the recall of windows R_ij is "the fraction
 * of detections computed by θ_best that are covered by rectangles in R_ij".  A detection
 * box counts as covered when it lies inside one window of its frame (reading R18).
 *   boxes [nb][5] int32 (frame, x0, y0, x1, y1), half-open, clipped to the frame;
 *   windows / frame_offset / frame_count as produced by otif_select_windows for n frames.
 * covered: device uint64, set to the number of covered boxes (enqueued; no sync). */
otif_status otif_window_recall(const int32_t *boxes, int64_t nb, const otif_window *windows,
                               const int32_t *frame_offset, const int32_t *frame_count, int32_t n,
                               unsigned long long *covered, cudaStream_t stream);

/* ---------------------------------------------------------------------------
 * §8(f) NEXT-3 — proxy training labels and training.
 * "at each 32 x 32 cell, the label is 1 if there is some detection d_i in D(t) that
 * intersects the cell, and 0 otherwise"; the model "should output a score
 * close to 1 at cells that intersect a detection, and 0 at other cells".
 * Loss: mean binary cross-entropy of sigmoid(z) over the cells of the batch (reading
 * R26); optimiser: Adam (reading R27).  Training arithmetic is fp32 (weights,
 * activations, gradients); reductions run in a fixed order (deterministic). */

/* Labels: boxes [nb][5] int32 (frame, x0, y0, x1, y1), half-open pixels; cell (cy, cx)
 * covers [cx*cell, (cx+1)*cell) x [cy*cell, (cy+1)*cell) clipped to the frame (R14).
 * labels [n][gh][gw] u8 (0/1), overwritten.  Boxes with a frame outside [0, n) or an
 * empty clipped area are ignored. */
otif_status otif_cell_labels(const int32_t *boxes, int64_t nb, int32_t n, int32_t gh, int32_t gw,
                             const otif_grid_desc *g, uint8_t *labels, cudaStream_t stream);

/* Adam step t >= 1 on fp32 device arrays (reading R27):
 * m = b1 m + (1-b1) g; v = b2 v + (1-b2) g^2; w -= lr (m/(1-b1^t)) / (sqrt(v/(1-b2^t)) + eps). */
otif_status otif_adam_step(float *w, float *m, float *v, const float *g, int64_t count, int32_t t, float lr,
                           float b1, float b2, float eps, cudaStream_t stream);

/* A trainer owns fp32 master weights (initialised from the host blob, layout as in
 * otif_proxy_create), Adam moments, gradients and the activations of up to max_batch
 * frames.  Any widths (enc[i] >= 1, 1 <= dec <= 256), n_strided 1..5. */
typedef struct otif_trainer otif_trainer;
otif_status otif_trainer_create(const otif_proxy_desc *d, const float *weights, size_t n_weights,
                                int32_t max_batch, otif_trainer **out);
void otif_trainer_destroy(otif_trainer *t);
/* Device views owned by the trainer: weights [n_weights], grads [n_weights]; output grid. */
otif_status otif_trainer_params(const otif_trainer *t, float **weights, float **grads, size_t *n_weights,
                                int32_t *gh, int32_t *gw);
/* Forward + loss + backward of one batch: img [n, in_h, in_w, 3] u8 (device), labels
 * [n, gh, gw] u8 (device) -> grads (overwritten), *loss = mean BCE (device float). */
otif_status otif_trainer_backward(otif_trainer *t, const uint8_t *img, const uint8_t *labels, int32_t n,
                                  float *loss, cudaStream_t stream);
/* One Adam step (b1 0.9, b2 0.999, eps 1e-8) of the master weights with the current
 * gradients; the step counter t is kept by the trainer. */
otif_status otif_trainer_adam(otif_trainer *t, float lr, cudaStream_t stream);

/* ---------------------------------------------------------------------------
 * §8(f) NEXT-4 — track refinement.  "we cluster tracks in S* prior to
 * inference, and construct a spatial index over cluster centers ... During inference,
 * we approximate the k-nearest neighbor lookup for a computed track s".
 * A track is a sequence of detection centres (reading R20):
 *   pts [total][2] float32 (x, y) in pixels, device; offsets [n+1] int64, device,
 *   track t = pts[offsets[t] .. offsets[t+1]), every track non-empty.
 * Resampled tracks P [n][npts][2] float32 (npts = N, 2 <= N <= 32; the paper uses
 * N = 20).  Coordinates must be finite.  Decisions (d <= eps, the k nearest)
 * are taken in fp32 with one IEEE rounding per operation in a fixed order (readings
 * R21–R25), so results are reproducible bit for bit.  All calls enqueue on `stream` and
 * do not synchronise; argument errors are reported synchronously (OTIF_EINVAL). */

/* P:L196 "we compute N points evenly spaced along each track": arc-length resampling,
 * endpoints included (reading R21).  P: caller-owned device [n][npts][2]. */
otif_status otif_track_resample(const float *pts, const int64_t *offsets, int64_t n, int32_t npts, float *P,
                                cudaStream_t stream);

/* P:L198 DBSCAN over S* with d(s1, s2) = (1/N) Σ_i eucl(P(s1)[i], P(s2)[i]):
 * neighbours d <= eps (a track neighbours itself), core iff >= min_pts neighbours,
 * clusters = connected components of core tracks numbered by their smallest index, a
 * border track joins the smallest-numbered cluster among its core neighbours, noise = -1
 * (reading R23: the classic algorithm run in index order).
 *   labels [n] int32, core [n] u8 (may be NULL), n_clusters: device int32 — all
 *   caller-owned device memory.  workspace >= otif_dbscan_workspace_bytes(n) (holds the
 *   n x n neighbour bitmap, n^2/8 bytes).  n <= 2^20. */
size_t otif_dbscan_workspace_bytes(int64_t n);
otif_status otif_track_dbscan(const float *P, int64_t n, int32_t npts, float eps, int32_t min_pts, int32_t *labels,
                              uint8_t *core, int32_t *n_clusters, void *workspace, size_t ws_bytes,
                              cudaStream_t stream);

/* P:L198 cluster centres: p_i = mean of {P(s)[i] | s in c}, summed in fp64 over the
 * members in index order, divided by the count, rounded to fp32.  nc = the host value of
 * n_clusters; labels outside [0, nc) are ignored.  centers [nc][npts][2] float32, sizes
 * [nc] int32: caller-owned device.  workspace >= otif_centers_workspace_bytes(n, nc). */
size_t otif_centers_workspace_bytes(int64_t n, int32_t nc);
otif_status otif_track_centers(const float *P, const int32_t *labels, int64_t n, int32_t npts, int32_t nc,
                               float *centers, int32_t *sizes, void *workspace, size_t ws_bytes,
                               cudaStream_t stream);

/* P:L200 refinement of m query tracks (raw pts/offsets as above): the candidate centres
 * pass within rho pixels of the first AND of the last detection (rho <= 0: all centres;
 * reading R24); the k closest candidates by (d, cluster index) are kept; start / end =
 * per-coordinate lower weighted median of the kept centres' first / last points with the
 * cluster sizes as weights (reading R25).  A track with no candidate keeps its own first
 * and last detection.  out [m][4] float32 (start x, start y, end x, end y), used [m]
 * int32 (clusters kept): caller-owned device.  1 <= k <= 16; the centres must fit in
 * shared memory next to the query buffers (nc <= 1000 at N = 20, else OTIF_EUNSUPPORTED). */
otif_status otif_track_refine(const float *pts, const int64_t *offsets, int64_t m, int32_t npts,
                              const float *centers, const int32_t *sizes, int32_t nc, int32_t k, float rho,
                              float *out, int32_t *used, cudaStream_t stream);

/* ---------------------------------------------------------------------------
 * Whole path on HOST frames (the end-to-end call): for batches of up to max_batch
 * frames, copy src (pinned or pageable host memory) to the device, run stages 1–5,
 * and copy the windows and per-frame counts back.  Two CUDA streams overlap the
 * host->device copy of batch b+1 with the compute of batch b.  The detector batches
 * stay on the device (the detector runs there); their per-size fill counts
 * are returned.
 *   desc: proxy shape (in_h/in_w = proxy resolution); src frames are src_h x src_w,
 *   the detector resolution is det_h x det_w; cell size, connectivity, W, threshold.
 * Results: windows_out [host, cap_windows], frame_count_out [host, n],
 * total_out [host], size_count_out [host, k] (all sizes accumulated over batches).
 * The call returns after the last copy completes (it synchronises its own streams). */
typedef struct {
    otif_proxy_desc proxy;
    int32_t src_h, src_w, det_h, det_w;
    otif_grid_desc grid;
    float threshold;
    int32_t k;
    otif_wsize sizes[8];
    int32_t max_batch;          /* frames per device batch (one select / pack launch each) */
    int32_t batch_cap[8];       /* detector batch capacity per size, per device batch */
    int32_t proxy_batch;        /* frames per resize + proxy launch within a batch (0 = max_batch) */
    int32_t pack_overlap;       /* stage 5 scheduling on device runs (identity crops, sizes with
                                   w*3 % 16 == 0; otherwise ignored):
                                   0 = pack each batch right after its selection;
                                   1 = the pack of batch b is copied by spare warps of batch b+1's
                                       tensor-bound proxy kernels (E4..D1, whose HBM is mostly idle),
                                       the remainder by a drain kernel; the last batch of a call is
                                       drained before the call returns;
                                   2 = as 1, and the last batch's pack also rides in the NEXT
                                       run_device call (or otif_pipeline_flush): its frames must stay
                                       valid until then.  Windows, counts and counters are final when
                                       the selection of a batch is; only the detector-batch bytes are
                                       deferred.  Host runs always use 0. */
} otif_pipeline_desc;

typedef struct otif_pipeline otif_pipeline;
otif_status otif_pipeline_create(const otif_pipeline_desc *d, const float *weights, size_t n_weights,
                                 otif_pipeline **out);
void otif_pipeline_destroy(otif_pipeline *p);
otif_status otif_pipeline_run_host(otif_pipeline *p, const uint8_t *src_host, int32_t n,
                                   otif_window *windows_out, int32_t cap_windows,
                                   int32_t *frame_count_out, int32_t *total_out,
                                   int32_t *size_count_out);
/* Same path on frames already resident in device memory, enqueued on `stream`
 * without any host synchronisation.  frame_base = global index of src_dev[0] (the
 * window hash keys windows by global frame, so a corpus sharded over ranks or clips
 * hashes identically).  Windows and detector batches of each device batch stay in
 * the pipeline's device buffers (overwritten batch by batch); the counters below
 * accumulate on the device across calls until reset. */
otif_status otif_pipeline_run_device(otif_pipeline *p, const uint8_t *src_dev, int32_t n, int64_t frame_base,
                                     cudaStream_t stream);
/* Device pointer to int64[15] counters accumulated since create/reset (run_host
 * resets them at its start): [0] frames, [1] positive cells, [2] windows, [3] window
 * pixels, [4] an order-independent hash of all windows (wrapping sum of 64-bit mixes
 * of (global frame, x, y, w, h, s)), [5 + s] windows of size s (8 slots), [13] windows
 * dropped because their slot exceeded batch_cap[s], [14] pixels of the windows packed. */
const int64_t *otif_pipeline_counters(const otif_pipeline *p);
/* Device pointers, valid after the last device batch's selection (stream order): per
 * frame of that batch (index = frame - batch start) the window-hash term (the sum of the
 * 64-bit mixes counter [4] accumulates; so a clip's hash is the wrapping sum over its
 * frames) and the window count. */
const int64_t *otif_pipeline_frame_hashes(const otif_pipeline *p);
const int32_t *otif_pipeline_frame_counts(const otif_pipeline *p);
/* Device pointer, valid after the last device batch's proxy (stream order): its cell
 * scores fp32 [n, gh, gw] (the proxy's score of every cell), index = frame -
 * batch start. */
const float *otif_pipeline_scores(const otif_pipeline *p);
/* Timing aid (otif_pipeline_set_timing on, pack_overlap > 0): pack copy units (P:L133's
 * crop/pack, in units of <= 32 KB of one window's rows) copied during each proxy GEMM layer
 * since the last call: units[0..4] = E2 (when not fused into E1+E2), E3, E4, E5, D1 (the
 * layers whose spare warps drain the previous batch's pack), units[5] = units left to the
 * drain kernel, units[6] = all units.  Synchronises the device; resets the tally. */
otif_status otif_pipeline_pack_units(otif_pipeline *p, uint64_t *units);
/* Device pointer to the detector batch of size s ([batch_cap[s], h_s, w_s, 3] u8, the
 * last packed device batch), or NULL. */
uint8_t *otif_pipeline_detector_batch(const otif_pipeline *p, int32_t s);
/* 1 if the last device batch skipped stage 1: the proxy's first kernel read the frames
 * itself (even integer downscale, the space-to-depth E1 variant), else 0. */
int32_t otif_pipeline_resize_fused(const otif_pipeline *p);
/* Complete a pack left pending by pack_overlap = 2 (enqueued on `stream`). */
otif_status otif_pipeline_flush(otif_pipeline *p, cudaStream_t stream);
otif_status otif_pipeline_reset_counters(otif_pipeline *p, cudaStream_t stream);
/* Per-stage device timing (CUDA events recorded between the stage launches on the
 * compute stream).  enable != 0 starts recording (and clears previous records). */
otif_status otif_pipeline_set_timing(otif_pipeline *p, int32_t enable);
/* Synchronises on the recorded events and returns the accumulated milliseconds per
 * stage since the last call: [0] resize, [1] proxy prep (workspace tag + E1),
 * [2..6] E2, E3, E4, E5, D1+D2 (the tcgen05 GEMM layers), [7] select (K5 + K6),
 * [8] pack (slots + copy), [9] append; n_ms >= 10.  *launches (optional) = kernels
 * launched by the pipeline since the last call. */
otif_status otif_pipeline_stage_ms(otif_pipeline *p, float *ms, int32_t n_ms, int64_t *launches);

#ifdef __cplusplus
}
#endif
#endif /* OTIF_H */
