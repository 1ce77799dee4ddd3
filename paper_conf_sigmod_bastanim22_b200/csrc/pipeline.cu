// pipeline.cu — the native runtime around the five stages (otif_pipeline_*): device
// buffers, a compute stream and a copy stream, the batch loop, and result accumulation.
//
// A device batch (max_batch frames) runs resize + proxy in mini-batches of proxy_batch
// frames, writing the scores of the whole batch; then one select launch and one pack
// launch cover the whole batch (the latency-bound grouping needs thousands of frames in
// flight to fill 148 SMs).  The detector batches stay on the device (the detector runs
// there); windows, per-frame counts and counters are accumulated on the device
// and copied back once per host call.  Host runs stage the frames of batch b+1 (copy
// stream, pinned host memory) while batch b computes.  Every stage is bracketed by an
// NVTX range (visible in nsys / ncu --nvtx) and, when timing is on, by CUDA events.
#include <nvtx3/nvToolsExt.h>
#include <stdlib.h>
#include <string.h>

#include <new>
#include <vector>

#include "common.cuh"
#include "packjob.cuh"

namespace otif {

otif_status launch_proxy(const otif_proxy *p, const uint8_t *img, int n, float *scores, uint8_t *ws, size_t ws_bytes,
                         cudaStream_t stream, cudaEvent_t *evs, PackJob *pj, const uint8_t *frames, int sh,
                         int sw, unsigned long long *pj_snap);
bool proxy_fuses_resize(const otif_proxy *p, int n, const uint8_t *src, int sh, int sw);
bool pack_job_applies(int32_t src_h, int32_t src_w, int32_t det_h, int32_t det_w, const otif_wsize *sizes, int32_t k,
                      uint8_t *const *batches);
otif_status launch_pack_prepare(const uint8_t *src, int32_t n, int32_t src_h, int32_t src_w,
                                const otif_window *windows, const int32_t *total, int32_t capacity,
                                const otif_wsize *sizes, int32_t k, uint8_t *const *batches, const int32_t *batch_cap,
                                int32_t *slot, int32_t *size_count, cudaStream_t stream, unsigned long long *ctr_pack,
                                PackJob *job_dev, int *inv);
otif_status launch_pack_units(PackJob *job_dev, cudaStream_t stream);
otif_status launch_select(const float *scores, const uint8_t *mask_in, float threshold, int32_t n, int32_t gh,
                          int32_t gw, const otif_grid_desc *g, const otif_wsize *sizes, int32_t k, uint8_t *mask_out,
                          otif_window *windows, int32_t capacity, int32_t *frame_count, int32_t *frame_offset,
                          int32_t *total, void *workspace, size_t ws_bytes, cudaStream_t stream,
                          unsigned long long *ctr, int frame_base, unsigned long long *est_sum,
                          unsigned long long *frame_hash);
otif_status launch_pack(const uint8_t *src, int32_t n, int32_t src_h, int32_t src_w, int32_t det_h, int32_t det_w,
                        const otif_window *windows, const int32_t *total, int32_t capacity, const otif_wsize *sizes,
                        int32_t k, uint8_t *const *batches, const int32_t *batch_cap, int32_t *slot,
                        int32_t *size_count, cudaStream_t stream, unsigned long long *ctr_pack);
int proxy_launches(const otif_proxy *p);

// timing stages: resize, proxy prep (tag + E1), E2, E3, E4, E5, D1+D2, select, pack, append
constexpr int kStages = 10;
enum { ST_START = -1, ST_RESIZE = 0, ST_PREP = 1, ST_SELECT = 7, ST_PACK = 8, ST_APPEND = 9 };

// counters (otif.h): [0] frames, [1] positive cells, [2] windows, [3] window pixels,
// [4] order-independent window hash, [5 + s] windows of size s (s < 8),
// [13] windows dropped for batch_cap, [14] pixels of the windows actually packed
constexpr int kCtrFixed = 5;
constexpr int kCtrPack = kCtrFixed + 8;
constexpr int kCtrTotal = kCtrPack + 2;

// Host runs only: append one batch's windows (frame index rebased to the global frame)
// and per-frame counts to the run's output arrays.  (The counters are accumulated by
// the select and slot kernels themselves.)
__global__ void __launch_bounds__(1024) append_kernel(const otif_window *__restrict__ win, const int *__restrict__ total,
                                                      int capacity, const int *__restrict__ counts, int nb,
                                                      int frame_base, otif_window *out_win, int out_cap,
                                                      int *out_counts, int *out_total) {
    const int t = min(*total, capacity);
    const int base = *out_total;
    for (int i = threadIdx.x; i < t; i += blockDim.x) {
        otif_window w = win[i];
        w.frame += frame_base;
        if (base + i < out_cap) out_win[base + i] = w;
    }
    for (int i = threadIdx.x; i < nb; i += blockDim.x) out_counts[frame_base + i] = counts[i];
    __syncthreads();
    if (threadIdx.x == 0) *out_total = base + *total;
}

}  // namespace otif

using namespace otif;

struct otif_pipeline {
    otif_pipeline_desc d;
    otif_proxy *proxy = nullptr;
    int gh = 0, gw = 0, cells = 0, cap_w = 0, pb = 0;
    uint8_t *src[2] = {nullptr, nullptr};   // host-run staging (allocated by the first host run)
    uint8_t *img = nullptr, *mask = nullptr, *proxy_ws = nullptr, *sel_ws = nullptr;
    size_t proxy_ws_bytes = 0, sel_ws_bytes = 0;
    float *scores = nullptr;
    otif_window *windows = nullptr;
    int *counts = nullptr, *offsets = nullptr, *total = nullptr, *slot = nullptr, *size_count = nullptr;
    unsigned long long *frame_hash = nullptr;   // per-frame window hash of the last device batch
    uint8_t *batches[8] = {};
    unsigned long long *ctr = nullptr;
    // run outputs of host calls (grown on demand)
    otif_window *out_win = nullptr;
    int out_win_cap = 0;
    int *out_counts = nullptr;
    int out_counts_cap = 0;
    int *out_total = nullptr;
    cudaStream_t s_compute = nullptr, s_copy = nullptr;
    cudaEvent_t ev_h2d[2] = {}, ev_free[2] = {};
    // optional per-stage timing: a log of spans (stage, start entry, end event); a span's
    // time is charged to its stage (stage < 0: a start marker)
    int timing = 0;
    std::vector<cudaEvent_t> ev_pool;
    std::vector<int> ev_stage, ev_from;
    size_t ev_used = 0;
    int64_t launches = 0;
    // pack overlap (desc.pack_overlap): the copy-unit queue of the last selected batch,
    // drained by the next batch's proxy kernels and pack_units_kernel
    PackJob *job = nullptr;
    int *inv = nullptr;
    int job_pending = 0;
    int resize_fused = 0;          // the last device batch read its frames in the proxy (no stage 1)
    cudaEvent_t ev_pending = nullptr;       // recorded where the pending job was built
    cudaStream_t pending_stream = nullptr;
    // timing only: per proxy pass that carried a pending job, the claim counter after each
    // GEMM layer [0..4] and the job's unit total [5] (device rows of 8, read by
    // otif_pipeline_pack_units)
    unsigned long long *pj_snaps = nullptr;
    int n_snaps = 0;
};
constexpr int kMaxSnaps = 1024;

// a pending job built on another stream: order this stream after it
static otif_status wait_pending(otif_pipeline *p, cudaStream_t st) {
    if (p->job_pending && st != p->pending_stream) OTIF_CUDA(cudaStreamWaitEvent(st, p->ev_pending, 0));
    return OTIF_OK;
}

// reserve a log entry (stage, from); its event is returned for the caller to record
static int treserve(otif_pipeline *p, int stage, int from, cudaEvent_t *ev) {
    if (p->ev_pool.size() <= p->ev_used) {
        cudaEvent_t e;
        if (cudaEventCreate(&e) != cudaSuccess) return -1;
        p->ev_pool.push_back(e);
        p->ev_stage.push_back(0);
        p->ev_from.push_back(-1);
    }
    p->ev_stage[p->ev_used] = stage;
    p->ev_from[p->ev_used] = from;
    *ev = p->ev_pool[p->ev_used];
    return (int)p->ev_used++;
}

// record a start marker on st; returns its entry (or -1 when timing is off)
static int tmark(otif_pipeline *p, cudaStream_t st) {
    if (!p->timing) return -1;
    cudaEvent_t e;
    int i = treserve(p, ST_START, -1, &e);
    if (i >= 0) cudaEventRecord(e, st);
    return i;
}

// close a span of `stage` opened at entry `from` (recorded on st); returns the new entry
static int tspan(otif_pipeline *p, int stage, cudaStream_t st, int from) {
    if (!p->timing || from < 0) return -1;
    cudaEvent_t e;
    int i = treserve(p, stage, from, &e);
    if (i >= 0) cudaEventRecord(e, st);
    return i;
}

#define RC(x)                           \
    do {                                \
        otif_status rc_ = (x);          \
        if (rc_ != OTIF_OK) return rc_; \
    } while (0)

// NVTX range for the host-side enqueue of one stage (nsys shows it on the CPU timeline
// and, with CUDA trace, correlates it with the stage's kernels)
struct NvtxRange {
    explicit NvtxRange(const char *name) { nvtxRangePushA(name); }
    ~NvtxRange() { nvtxRangePop(); }
};

static otif_status run_proxy(otif_pipeline *p, const uint8_t *img, int mb, float *scores, cudaStream_t st,
                             PackJob *pj, const uint8_t *frames) {
    NvtxRange r("otif.proxy");
    // six spans for the proxy (prep/E1, then each GEMM layer); launch_proxy records their
    // end events at the actual points in the stream
    cudaEvent_t evs[6];
    int from = tmark(p, st);
    for (int i = 0; i < 6 && p->timing; i++) from = treserve(p, ST_PREP + i, from, &evs[i]);
    unsigned long long *snap = nullptr;
    if (p->timing && pj && p->n_snaps < kMaxSnaps) {
        if (!p->pj_snaps && cudaMalloc(&p->pj_snaps, (size_t)kMaxSnaps * 8 * 8) != cudaSuccess) return OTIF_ENOMEM;
        snap = p->pj_snaps + (size_t)p->n_snaps++ * 8;
        OTIF_CUDA(cudaMemsetAsync(snap, 0, 8 * 8, st));   // layers without a GEMM launch stay 0
        OTIF_CUDA(cudaMemcpyAsync(snap + 5, &pj->units_base[p->d.k], 8, cudaMemcpyDeviceToDevice, st));
    }
    RC(launch_proxy(p->proxy, img, mb, scores, p->proxy_ws, p->proxy_ws_bytes, st, p->timing ? evs : nullptr, pj,
                    frames, p->d.src_h, p->d.src_w, snap));
    p->launches += proxy_launches(p->proxy);
    return OTIF_OK;
}

// drain the pending pack job (whatever the fused copy warps did not take)
static otif_status drain_pack(otif_pipeline *p, cudaStream_t st) {
    if (!p->job_pending) return OTIF_OK;
    RC(wait_pending(p, st));
    NvtxRange r("otif.pack_drain");
    int t0 = tmark(p, st);
    RC(launch_pack_units(p->job, st));
    tspan(p, ST_PACK, st, t0);
    p->launches += 1;
    p->job_pending = 0;
    return OTIF_OK;
}

// overlap: 0 = pack right after select; 1 = leave the pack pending for the next batch's
// proxy (the caller drains it at the end of the call or keeps it for the next call)
static otif_status run_batch(otif_pipeline *p, const uint8_t *src, int nb, int frame_base, cudaStream_t st,
                             int overlap) {
    const otif_pipeline_desc &d = p->d;
    const size_t frame_bytes = (size_t)d.src_h * d.src_w * 3;
    RC(wait_pending(p, st));
    for (int m0 = 0; m0 < nb; m0 += p->pb) {
        const int mb = nb - m0 < p->pb ? nb - m0 : p->pb;
        const uint8_t *frames = src + (size_t)m0 * frame_bytes;
        // even integer downscale: the fused E1+E2 kernel reads the frames itself (stage 1
        // fused into the proxy's first kernel, no proxy image in HBM)
        const bool fused = proxy_fuses_resize(p->proxy, mb, frames, d.src_h, d.src_w);
        p->resize_fused = fused ? 1 : 0;
        {
            NvtxRange r("otif.resize");
            int t0 = tmark(p, st);
            if (!fused) {
                RC(otif_resize(frames, mb, d.src_h, d.src_w, p->img, d.proxy.in_h, d.proxy.in_w, st));
                p->launches += 1;
            }
            tspan(p, ST_RESIZE, st, t0);
        }
        // the pending pack (previous batch) rides in this proxy pass's tensor-bound layers
        RC(run_proxy(p, p->img, mb, p->scores + (size_t)m0 * p->cells, st, p->job_pending ? p->job : nullptr,
                     fused ? frames : nullptr));
    }
    RC(drain_pack(p, st));
    {
        NvtxRange r("otif.select");
        int t0 = tmark(p, st);
        RC(launch_select(p->scores, nullptr, d.threshold, nb, p->gh, p->gw, &d.grid, d.sizes, d.k, p->mask, p->windows,
                         p->cap_w, p->counts, p->offsets, p->total, p->sel_ws, p->sel_ws_bytes, st, p->ctr, frame_base,
                         nullptr, p->frame_hash));
        tspan(p, ST_SELECT, st, t0);
        p->launches += 2;
    }
    NvtxRange r("otif.pack");
    int t0 = tmark(p, st);
    if (overlap && p->job) {
        RC(launch_pack_prepare(src, nb, d.src_h, d.src_w, p->windows, p->total, p->cap_w, d.sizes, d.k, p->batches,
                               d.batch_cap, p->slot, p->size_count, st, p->ctr + kCtrPack, p->job, p->inv));
        p->job_pending = 1;
        p->pending_stream = st;
        OTIF_CUDA(cudaEventRecord(p->ev_pending, st));
        p->launches += 1;
    } else {
        RC(launch_pack(src, nb, d.src_h, d.src_w, d.det_h, d.det_w, p->windows, p->total, p->cap_w, d.sizes, d.k,
                       p->batches, d.batch_cap, p->slot, p->size_count, st, p->ctr + kCtrPack));
        p->launches += 2;
    }
    t0 = tspan(p, ST_PACK, st, t0);
    if (p->out_win) {
        append_kernel<<<1, 1024, 0, st>>>(p->windows, p->total, p->cap_w, p->counts, nb, frame_base, p->out_win,
                                          p->out_win_cap, p->out_counts, p->out_total);
        OTIF_LAUNCH_CHECK();
        p->launches += 1;
        tspan(p, ST_APPEND, st, t0);
    }
    return OTIF_OK;
}

#define PCUDA(call)                                                                    \
    do {                                                                               \
        cudaError_t e_ = (call);                                                       \
        if (e_ != cudaSuccess) {                                                       \
            set_error("%s: %s", #call, cudaGetErrorString(e_));                        \
            otif_pipeline_destroy(p);                                                  \
            return e_ == cudaErrorMemoryAllocation ? OTIF_ENOMEM : OTIF_ECUDA;         \
        }                                                                              \
    } while (0)

extern "C" otif_status otif_pipeline_create(const otif_pipeline_desc *d, const float *weights, size_t n_weights,
                                            otif_pipeline **out) {
    OTIF_REQUIRE(d && weights && out, "otif_pipeline_create: NULL argument");
    OTIF_REQUIRE(d->max_batch > 0, "otif_pipeline_create: max_batch must be positive");
    OTIF_REQUIRE(d->proxy_batch >= 0, "otif_pipeline_create: proxy_batch must be >= 0");
    OTIF_REQUIRE(d->k >= 1 && d->k <= 8, "otif_pipeline_create: k=%d", d->k);
    OTIF_REQUIRE(d->src_h > 0 && d->src_w > 0 && d->det_h > 0 && d->det_w > 0, "otif_pipeline_create: sizes");
    OTIF_REQUIRE(d->grid.frame_w == d->det_w && d->grid.frame_h == d->det_h,
                 "otif_pipeline_create: grid frame must be the detector resolution");
    for (int s = 0; s < d->k; s++) OTIF_REQUIRE(d->batch_cap[s] >= 0, "otif_pipeline_create: batch_cap[%d] < 0", s);
    OTIF_REQUIRE(d->pack_overlap >= 0 && d->pack_overlap <= 2, "otif_pipeline_create: pack_overlap %d", d->pack_overlap);
    otif_pipeline *p = new (std::nothrow) otif_pipeline();
    if (!p) return OTIF_ENOMEM;
    p->d = *d;
    otif_status rc = otif_proxy_create(&d->proxy, weights, n_weights, &p->proxy);
    if (rc != OTIF_OK) { otif_pipeline_destroy(p); return rc; }
    otif_proxy_grid(p->proxy, &p->gh, &p->gw);
    if (p->gh != (d->grid.frame_h + d->grid.cell - 1) / d->grid.cell ||
        p->gw != (d->grid.frame_w + d->grid.cell - 1) / d->grid.cell) {
        set_error("otif_pipeline_create: proxy grid %dx%d does not match ceil(frame/cell)", p->gw, p->gh);
        otif_pipeline_destroy(p);
        return OTIF_EINVAL;
    }
    const int B = d->max_batch;
    p->pb = (d->proxy_batch > 0 && d->proxy_batch < B) ? d->proxy_batch : B;
    p->cells = p->gh * p->gw;
    p->cap_w = B * ((p->cells + 1) / 2);
    PCUDA(cudaMalloc(&p->img, (size_t)p->pb * d->proxy.in_h * d->proxy.in_w * 3));
    p->proxy_ws_bytes = otif_proxy_workspace_bytes(p->proxy, p->pb);
    PCUDA(cudaMalloc(&p->proxy_ws, p->proxy_ws_bytes));
    PCUDA(cudaMemset(p->proxy_ws, 0, p->proxy_ws_bytes));
    p->sel_ws_bytes = otif_select_workspace_bytes(B, p->gh, p->gw);
    PCUDA(cudaMalloc(&p->sel_ws, p->sel_ws_bytes));
    PCUDA(cudaMalloc(&p->scores, (size_t)B * p->cells * 4));
    PCUDA(cudaMalloc(&p->mask, (size_t)B * p->cells));
    PCUDA(cudaMalloc(&p->windows, (size_t)p->cap_w * sizeof(otif_window)));
    PCUDA(cudaMalloc(&p->counts, B * 4));
    PCUDA(cudaMalloc(&p->frame_hash, (size_t)B * 8));
    PCUDA(cudaMalloc(&p->offsets, B * 4));
    PCUDA(cudaMalloc(&p->total, 4));
    PCUDA(cudaMalloc(&p->slot, (size_t)p->cap_w * 4));
    PCUDA(cudaMalloc(&p->size_count, 8 * 4));
    for (int s = 0; s < d->k; s++)
        if (d->batch_cap[s] > 0)
            PCUDA(cudaMalloc(&p->batches[s], (size_t)d->batch_cap[s] * d->sizes[s].w * d->sizes[s].h * 3));
    if (d->pack_overlap && pack_job_applies(d->src_h, d->src_w, d->det_h, d->det_w, d->sizes, d->k, p->batches)) {
        int64_t inv_n = 0;
        for (int s = 0; s < d->k; s++) inv_n += d->batch_cap[s];
        PCUDA(cudaMalloc(&p->job, sizeof(PackJob)));
        PCUDA(cudaEventCreateWithFlags(&p->ev_pending, cudaEventDisableTiming));
        PCUDA(cudaMalloc(&p->inv, (size_t)(inv_n > 0 ? inv_n : 1) * 4));
    }
    PCUDA(cudaMalloc(&p->ctr, kCtrTotal * 8));
    PCUDA(cudaMemset(p->ctr, 0, kCtrTotal * 8));
    PCUDA(cudaMalloc(&p->out_total, 4));
    PCUDA(cudaStreamCreateWithFlags(&p->s_compute, cudaStreamNonBlocking));
    PCUDA(cudaStreamCreateWithFlags(&p->s_copy, cudaStreamNonBlocking));
    for (int i = 0; i < 2; i++) {
        PCUDA(cudaEventCreateWithFlags(&p->ev_h2d[i], cudaEventDisableTiming));
        PCUDA(cudaEventCreateWithFlags(&p->ev_free[i], cudaEventDisableTiming));
    }
    PCUDA(cudaDeviceSynchronize());
    *out = p;
    return OTIF_OK;
}

extern "C" void otif_pipeline_destroy(otif_pipeline *p) {
    if (!p) return;
    if (p->job_pending && p->pending_stream) cudaStreamSynchronize(p->pending_stream);
    if (p->s_compute) cudaStreamSynchronize(p->s_compute);
    if (p->s_copy) cudaStreamSynchronize(p->s_copy);
    void *bufs[] = {p->src[0], p->src[1], p->img, p->mask, p->proxy_ws, p->sel_ws, p->scores, p->windows, p->counts,
                    p->offsets, p->total, p->slot, p->size_count, p->ctr, p->out_win, p->out_counts, p->out_total,
                    p->job, p->inv, p->frame_hash, p->pj_snaps};
    for (void *b : bufs)
        if (b) cudaFree(b);
    for (int s = 0; s < 8; s++)
        if (p->batches[s]) cudaFree(p->batches[s]);
    for (cudaEvent_t e : p->ev_pool) cudaEventDestroy(e);
    if (p->ev_pending) cudaEventDestroy(p->ev_pending);
    for (int i = 0; i < 2; i++) {
        if (p->ev_h2d[i]) cudaEventDestroy(p->ev_h2d[i]);
        if (p->ev_free[i]) cudaEventDestroy(p->ev_free[i]);
    }
    if (p->s_compute) cudaStreamDestroy(p->s_compute);
    if (p->s_copy) cudaStreamDestroy(p->s_copy);
    if (p->proxy) otif_proxy_destroy(p->proxy);
    delete p;
}

static otif_status ensure_outputs(otif_pipeline *p, int n, int cap_windows) {
    if (!p->src[0]) {   // double-buffered host staging, first host run only
        const size_t bytes = (size_t)p->d.max_batch * p->d.src_h * p->d.src_w * 3;
        OTIF_CUDA(cudaMalloc(&p->src[0], bytes));
        OTIF_CUDA(cudaMalloc(&p->src[1], bytes));
    }
    if (n > p->out_counts_cap) {
        if (p->out_counts) cudaFree(p->out_counts);
        p->out_counts = nullptr;
        OTIF_CUDA(cudaMalloc(&p->out_counts, (size_t)n * 4));
        p->out_counts_cap = n;
    }
    if (cap_windows > p->out_win_cap) {
        if (p->out_win) cudaFree(p->out_win);
        p->out_win = nullptr;
        OTIF_CUDA(cudaMalloc(&p->out_win, (size_t)cap_windows * sizeof(otif_window)));
        p->out_win_cap = cap_windows;
    }
    return OTIF_OK;
}

extern "C" otif_status otif_pipeline_run_host(otif_pipeline *p, const uint8_t *src_host, int32_t n,
                                              otif_window *windows_out, int32_t cap_windows, int32_t *frame_count_out,
                                              int32_t *total_out, int32_t *size_count_out) {
    OTIF_REQUIRE(p && (src_host || n == 0) && n >= 0 && cap_windows >= 0, "otif_pipeline_run_host: bad arguments");
    OTIF_REQUIRE(total_out, "otif_pipeline_run_host: NULL total_out");
    NvtxRange range("otif.pipeline_run_host");
    RC(ensure_outputs(p, n > 0 ? n : 1, cap_windows > 0 ? cap_windows : 1));
    const otif_pipeline_desc &d = p->d;
    const size_t frame_bytes = (size_t)d.src_h * d.src_w * 3;
    RC(drain_pack(p, p->s_compute));   // a pack left pending by a device run (same frames lifetime rule)
    OTIF_CUDA(cudaMemsetAsync(p->out_total, 0, 4, p->s_compute));
    OTIF_CUDA(cudaMemsetAsync(p->ctr, 0, kCtrTotal * 8, p->s_compute));
    // the copy stream must not overwrite a src buffer before the compute stream is done with it
    for (int i = 0; i < 2; i++) OTIF_CUDA(cudaEventRecord(p->ev_free[i], p->s_compute));
    const int cap_saved = p->out_win_cap;
    p->out_win_cap = cap_windows;  // windows beyond the caller's capacity are dropped (total stays exact)
    otif_status rc = OTIF_OK;
    int b = 0;
    for (int f0 = 0; f0 < n && rc == OTIF_OK; f0 += d.max_batch, b++) {
        const int nb = n - f0 < d.max_batch ? n - f0 : d.max_batch;
        const int buf = b & 1;
        OTIF_CUDA(cudaStreamWaitEvent(p->s_copy, p->ev_free[buf], 0));
        OTIF_CUDA(cudaMemcpyAsync(p->src[buf], src_host + (size_t)f0 * frame_bytes, (size_t)nb * frame_bytes,
                                  cudaMemcpyHostToDevice, p->s_copy));
        OTIF_CUDA(cudaEventRecord(p->ev_h2d[buf], p->s_copy));
        OTIF_CUDA(cudaStreamWaitEvent(p->s_compute, p->ev_h2d[buf], 0));
        rc = run_batch(p, p->src[buf], nb, f0, p->s_compute, 0);   // host runs are PCIe-bound: no pack overlap
        if (rc == OTIF_OK) OTIF_CUDA(cudaEventRecord(p->ev_free[buf], p->s_compute));
    }
    p->out_win_cap = cap_saved;
    if (rc != OTIF_OK) return rc;
    int total = 0;
    OTIF_CUDA(cudaMemcpyAsync(&total, p->out_total, 4, cudaMemcpyDeviceToHost, p->s_compute));
    if (frame_count_out && n > 0)
        OTIF_CUDA(cudaMemcpyAsync(frame_count_out, p->out_counts, (size_t)n * 4, cudaMemcpyDeviceToHost, p->s_compute));
    unsigned long long ctr[kCtrTotal];
    OTIF_CUDA(cudaMemcpyAsync(ctr, p->ctr, sizeof(ctr), cudaMemcpyDeviceToHost, p->s_compute));
    OTIF_CUDA(cudaStreamSynchronize(p->s_compute));
    const int keep = total < cap_windows ? total : cap_windows;
    if (windows_out && keep > 0)
        OTIF_CUDA(cudaMemcpy(windows_out, p->out_win, (size_t)keep * sizeof(otif_window), cudaMemcpyDeviceToHost));
    *total_out = total;
    if (size_count_out)
        for (int s = 0; s < d.k; s++) size_count_out[s] = (int32_t)ctr[kCtrFixed + s];
    return OTIF_OK;
}

extern "C" otif_status otif_pipeline_run_device(otif_pipeline *p, const uint8_t *src_dev, int32_t n,
                                                int64_t frame_base, cudaStream_t stream) {
    OTIF_REQUIRE(p && (src_dev || n == 0) && n >= 0 && frame_base >= 0 && frame_base + n < (1ll << 31),
                 "otif_pipeline_run_device: bad arguments");
    NvtxRange range("otif.pipeline_run_device");
    const size_t frame_bytes = (size_t)p->d.src_h * p->d.src_w * 3;
    // device runs keep no per-frame outputs beyond the current batch: counters only
    otif_window *ow = p->out_win;
    int *oc = p->out_counts;
    p->out_win = nullptr;
    p->out_counts = nullptr;
    otif_status rc = OTIF_OK;
    for (int f0 = 0; f0 < n && rc == OTIF_OK; f0 += p->d.max_batch) {
        const int nb = n - f0 < p->d.max_batch ? n - f0 : p->d.max_batch;
        rc = run_batch(p, src_dev + (size_t)f0 * frame_bytes, nb, (int)(frame_base + f0), stream,
                       p->d.pack_overlap != 0);
    }
    // pack_overlap 1: the last batch's pack completes within this call; 2: it stays pending
    // for the next call's proxy (or otif_pipeline_flush)
    if (rc == OTIF_OK && p->d.pack_overlap == 1) rc = drain_pack(p, stream);
    p->out_win = ow;
    p->out_counts = oc;
    return rc;
}

extern "C" const int64_t *otif_pipeline_frame_hashes(const otif_pipeline *p) {
    return p ? reinterpret_cast<const int64_t *>(p->frame_hash) : nullptr;
}

extern "C" const int32_t *otif_pipeline_frame_counts(const otif_pipeline *p) {
    return p ? p->counts : nullptr;
}

extern "C" const float *otif_pipeline_scores(const otif_pipeline *p) {
    return p ? p->scores : nullptr;
}

extern "C" otif_status otif_pipeline_pack_units(otif_pipeline *p, uint64_t *units) {
    OTIF_REQUIRE(p && units, "otif_pipeline_pack_units: NULL argument");
    for (int i = 0; i < 7; i++) units[i] = 0;
    if (p->n_snaps > 0) {
        std::vector<unsigned long long> h((size_t)p->n_snaps * 8);
        OTIF_CUDA(cudaMemcpy(h.data(), p->pj_snaps, h.size() * 8, cudaMemcpyDeviceToHost));
        for (int c = 0; c < p->n_snaps; c++) {
            const unsigned long long *r = &h[(size_t)c * 8];
            const unsigned long long tot = r[5];
            unsigned long long prev = 0;
            for (int li = 0; li < 5; li++) {
                // (a pass without an E2 GEMM layer never writes slot 0: it stays 0)
                const unsigned long long cur = r[li] < tot ? r[li] : tot;
                if (cur >= prev) { units[li] += cur - prev; prev = cur; }
            }
            units[5] += tot - prev;   // left to the drain kernel
            units[6] += tot;
        }
    }
    p->n_snaps = 0;
    return OTIF_OK;
}

extern "C" uint8_t *otif_pipeline_detector_batch(const otif_pipeline *p, int32_t s) {
    return (p && s >= 0 && s < p->d.k) ? p->batches[s] : nullptr;
}

extern "C" int32_t otif_pipeline_resize_fused(const otif_pipeline *p) { return p ? p->resize_fused : 0; }

extern "C" otif_status otif_pipeline_flush(otif_pipeline *p, cudaStream_t stream) {
    OTIF_REQUIRE(p, "otif_pipeline_flush: NULL");
    return drain_pack(p, stream);
}

extern "C" const int64_t *otif_pipeline_counters(const otif_pipeline *p) {
    return p ? reinterpret_cast<const int64_t *>(p->ctr) : nullptr;
}

extern "C" otif_status otif_pipeline_reset_counters(otif_pipeline *p, cudaStream_t stream) {
    OTIF_REQUIRE(p, "otif_pipeline_reset_counters: NULL");
    OTIF_CUDA(cudaMemsetAsync(p->ctr, 0, kCtrTotal * 8, stream));
    return OTIF_OK;
}

extern "C" otif_status otif_pipeline_set_timing(otif_pipeline *p, int32_t enable) {
    OTIF_REQUIRE(p, "otif_pipeline_set_timing: NULL");
    p->timing = enable ? 1 : 0;
    p->ev_used = 0;
    p->launches = 0;
    p->n_snaps = 0;
    // the pack-unit snapshot rows are allocated here, not inside a timed run
    if (p->timing && p->job && !p->pj_snaps && cudaMalloc(&p->pj_snaps, (size_t)kMaxSnaps * 8 * 8) != cudaSuccess)
        return OTIF_ENOMEM;
    return OTIF_OK;
}

extern "C" otif_status otif_pipeline_stage_ms(otif_pipeline *p, float *ms, int32_t n_ms, int64_t *launches) {
    OTIF_REQUIRE(p && ms && n_ms >= kStages, "otif_pipeline_stage_ms: need %d entries", kStages);
    for (int s = 0; s < kStages; s++) ms[s] = 0.0f;
    if (p->ev_used > 0) OTIF_CUDA(cudaEventSynchronize(p->ev_pool[p->ev_used - 1]));
    for (size_t i = 0; i < p->ev_used; i++) {
        const int s = p->ev_stage[i], from = p->ev_from[i];
        if (s < 0 || from < 0) continue;  // a start marker: no time charged
        float t = 0.0f;
        OTIF_CUDA(cudaEventElapsedTime(&t, p->ev_pool[from], p->ev_pool[i]));
        ms[s] += t;
    }
    if (launches) *launches = p->launches;
    p->ev_used = 0;
    p->launches = 0;
    return OTIF_OK;
}
