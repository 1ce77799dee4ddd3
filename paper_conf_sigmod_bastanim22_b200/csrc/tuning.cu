// tuning.cu — §8(f) NEXT rows built on the stage-4 kernels.
//
// NEXT-1 otif_choose_window_sizes: greedy choice of the fixed window-size
//   set W over perfect-proxy masks.  Every candidate of a round is scored by one launch of
//   the select kernel over all frames accumulating Σ_t est(R_t) on the device; one
//   device->host copy per round picks the greatest decrease.
// NEXT-2 otif_window_recall: the recall numerator of the proxy-tuning sweep —
//   one thread per detection box tests containment in the windows of its frame.
#include <string.h>

#include <vector>

#include "common.cuh"

namespace otif {

otif_status launch_select(const float *scores, const uint8_t *mask_in, float threshold, int32_t n, int32_t gh,
                          int32_t gw, const otif_grid_desc *g, const otif_wsize *sizes, int32_t k, uint8_t *mask_out,
                          otif_window *windows, int32_t capacity, int32_t *frame_count, int32_t *frame_offset,
                          int32_t *total, void *workspace, size_t ws_bytes, cudaStream_t stream,
                          unsigned long long *ctr, int frame_base, unsigned long long *est_sum);
otif_status validate_select(const float *scores, const uint8_t *mask_in, int32_t n, int32_t gh, int32_t gw,
                            const otif_grid_desc *g, const otif_wsize *sizes, int32_t k, int32_t capacity);
size_t select_workspace_bytes(int32_t n, int32_t gh, int32_t gw);

__global__ void covered_kernel(const int32_t *__restrict__ boxes, int64_t nb, const otif_window *__restrict__ win,
                               const int32_t *__restrict__ frame_offset, const int32_t *__restrict__ frame_count,
                               int32_t n, unsigned long long *covered) {
    unsigned long long mine = 0;
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < nb; i += (int64_t)gridDim.x * blockDim.x) {
        const int32_t *b = boxes + i * 5;
        const int f = b[0];
        if (f < 0 || f >= n) continue;
        const int o = frame_offset[f], c = frame_count[f];
        for (int g = o; g < o + c; g++) {
            const otif_window w = win[g];
            if (w.x <= b[1] && b[3] <= w.x + w.w && w.y <= b[2] && b[4] <= w.y + w.h) { mine++; break; }
        }
    }
    for (int s = 16; s > 0; s >>= 1) mine += __shfl_xor_sync(0xffffffffu, mine, s);
    if ((threadIdx.x & 31) == 0 && mine) atomicAdd(covered, mine);
}

}  // namespace otif

using namespace otif;

extern "C" size_t otif_choose_workspace_bytes(int32_t n, int32_t gh, int32_t gw, int32_t m) {
    if (n < 0 || gh <= 0 || gw <= 0 || m < 0) return 0;
    const size_t cap = (size_t)n * ((gh * gw + 1) / 2 > 1 ? (gh * gw + 1) / 2 : 1);
    return select_workspace_bytes(n, gh, gw) + round_up((int64_t)(m + 1) * 8, 256) +
           round_up((int64_t)cap * sizeof(otif_window), 256) + 3 * round_up((int64_t)n * 4 + 4, 256);
}

extern "C" otif_status otif_choose_window_sizes(const uint8_t *masks, int32_t n, int32_t gh, int32_t gw,
                                                const otif_grid_desc *g, const otif_wsize *candidates, int32_t m,
                                                int64_t full_cost, int32_t k, int32_t *chosen_idx, int64_t *est,
                                                void *workspace, size_t ws_bytes, cudaStream_t stream) {
    OTIF_REQUIRE(g && (candidates || m == 0) && chosen_idx && est, "otif_choose_window_sizes: NULL argument");
    OTIF_REQUIRE(k >= 1 && k <= 8 && m >= 0 && n >= 0, "otif_choose_window_sizes: k=%d m=%d n=%d", k, m, n);
    OTIF_REQUIRE(n == 0 || (masks && workspace), "otif_choose_window_sizes: NULL masks/workspace");
    OTIF_REQUIRE(ws_bytes >= otif_choose_workspace_bytes(n, gh, gw, m), "otif_choose_window_sizes: workspace too small");
    otif_wsize W[8];
    W[0].w = g->frame_w; W[0].h = g->frame_h; W[0].cost = full_cost;
    otif_status st = validate_select(nullptr, masks ? masks : (const uint8_t *)1, n, gh, gw, g, W, 1, 0);
    if (st != OTIF_OK) return st;
    for (int c = 0; c < m; c++)
        OTIF_REQUIRE(candidates[c].w > 0 && candidates[c].h > 0 && candidates[c].w <= g->frame_w &&
                         candidates[c].h <= g->frame_h,
                     "otif_choose_window_sizes: candidate %d (%dx%d) not inside the frame", c, candidates[c].w,
                     candidates[c].h);
    st = check_device(nullptr);
    if (st != OTIF_OK) return st;
    // workspace: [select ws][est sums (m+1) int64][windows][counts][offsets][total]
    uint8_t *ws = (uint8_t *)workspace;
    const size_t sel_bytes = select_workspace_bytes(n, gh, gw);
    unsigned long long *sums = (unsigned long long *)(ws + sel_bytes);
    const size_t cap = (size_t)n * ((gh * gw + 1) / 2 > 1 ? (gh * gw + 1) / 2 : 1);
    otif_window *win = (otif_window *)(ws + sel_bytes + round_up((int64_t)(m + 1) * 8, 256));
    int32_t *cnt = (int32_t *)((uint8_t *)win + round_up((int64_t)cap * sizeof(otif_window), 256));
    int32_t *off = (int32_t *)((uint8_t *)cnt + round_up((int64_t)n * 4 + 4, 256));
    int32_t *tot = (int32_t *)((uint8_t *)off + round_up((int64_t)n * 4 + 4, 256));

    std::vector<unsigned long long> h(m + 1);
    std::vector<char> used(m > 0 ? m : 1, 0);
    int nw = 1;
    // Σ est with W = {full frame}
    OTIF_CUDA(cudaMemsetAsync(sums, 0, (m + 1) * 8, stream));
    if (n > 0) {
        st = launch_select(nullptr, masks, 0.0f, n, gh, gw, g, W, 1, nullptr, win, 0, cnt, off, tot, ws, sel_bytes,
                           stream, nullptr, 0, sums + m);
        if (st != OTIF_OK) return st;
    }
    OTIF_CUDA(cudaMemcpyAsync(&h[m], sums + m, 8, cudaMemcpyDeviceToHost, stream));
    OTIF_CUDA(cudaStreamSynchronize(stream));
    chosen_idx[0] = -1;
    est[0] = (int64_t)h[m];
    int64_t cur = est[0];
    while (nw < k) {
        OTIF_CUDA(cudaMemsetAsync(sums, 0, m * 8, stream));
        for (int c = 0; c < m && n > 0; c++) {
            if (used[c]) continue;
            W[nw] = candidates[c];
            st = launch_select(nullptr, masks, 0.0f, n, gh, gw, g, W, nw + 1, nullptr, win, 0, cnt, off, tot, ws,
                               sel_bytes, stream, nullptr, 0, sums + c);
            if (st != OTIF_OK) return st;
        }
        if (m > 0) OTIF_CUDA(cudaMemcpyAsync(h.data(), sums, m * 8, cudaMemcpyDeviceToHost, stream));
        OTIF_CUDA(cudaStreamSynchronize(stream));
        int best = -1;
        int64_t best_sum = cur;
        for (int c = 0; c < m; c++) {
            if (used[c]) continue;
            const int64_t s = n > 0 ? (int64_t)h[c] : 0;
            if (s < best_sum) { best_sum = s; best = c; }  // greatest decrease; ties: earliest candidate
        }
        if (best < 0) break;  // no candidate decreases the sum (reading R19)
        used[best] = 1;
        W[nw] = candidates[best];
        chosen_idx[nw] = best;
        est[nw] = best_sum;
        cur = best_sum;
        nw++;
    }
    for (int i = nw; i < k; i++) { chosen_idx[i] = -2; est[i] = cur; }
    return OTIF_OK;
}

extern "C" otif_status otif_window_recall(const int32_t *boxes, int64_t nb, const otif_window *windows,
                                          const int32_t *frame_offset, const int32_t *frame_count, int32_t n,
                                          unsigned long long *covered, cudaStream_t stream) {
    OTIF_REQUIRE(nb >= 0 && n >= 0 && covered, "otif_window_recall: bad arguments");
    OTIF_REQUIRE(nb == 0 || (boxes && windows && frame_offset && frame_count), "otif_window_recall: NULL pointer");
    int num_sms = 148;
    otif_status st = check_device(&num_sms);
    if (st != OTIF_OK) return st;
    OTIF_CUDA(cudaMemsetAsync(covered, 0, 8, stream));
    if (nb == 0) return OTIF_OK;
    int64_t blocks = cdiv(nb, 256);
    if (blocks > num_sms * 8) blocks = num_sms * 8;
    covered_kernel<<<(unsigned)blocks, 256, 0, stream>>>(boxes, nb, windows, frame_offset, frame_count, n, covered);
    OTIF_LAUNCH_CHECK();
    return OTIF_OK;
}
