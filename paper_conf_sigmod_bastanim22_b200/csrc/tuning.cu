// tuning.cu — §8(f) NEXT rows built on the stage-4 kernels.
//
// NEXT-1 otif_choose_window_sizes: greedy choice of the fixed window-size
//   set W over perfect-proxy masks.  Each round scores EVERY remaining candidate in one
//   launch of the grouping kernel (grid.y = candidate: warp per (frame, candidate),
//   Σ_t est(R_t) accumulated per candidate on the device); one device->host copy per
//   round picks the greatest decrease.
// NEXT-2 otif_window_recall: the recall numerator of the proxy-tuning sweep —
//   one thread per detection box tests containment in the windows of its frame.
#include <string.h>

#include <vector>

#include "common.cuh"

namespace otif {

otif_status validate_select(const float *scores, const uint8_t *mask_in, int32_t n, int32_t gh, int32_t gw,
                            const otif_grid_desc *g, const otif_wsize *sizes, int32_t k, int32_t capacity);
otif_status launch_select_multi(const uint8_t *masks, int32_t n, int32_t gh, int32_t gw, const otif_grid_desc *g,
                                const otif_wsize *const *sets, const int32_t *set_k, int32_t m, void *wtab_dev,
                                unsigned long long *est_sums, cudaStream_t stream);
constexpr size_t kWTableBytes = 192;   // >= sizeof(WTable) (static_assert in select.cu)

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
    // [W' tables (m + 1)][est sums (m + 1) int64]
    return round_up((int64_t)(m + 1) * kWTableBytes, 256) + round_up((int64_t)(m + 1) * 8, 256);
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
    uint8_t *ws = (uint8_t *)workspace;
    void *wtab = ws;
    unsigned long long *sums = (unsigned long long *)(ws + round_up((int64_t)(m + 1) * kWTableBytes, 256));

    std::vector<unsigned long long> h(m + 1, 0);
    std::vector<char> used(m > 0 ? m : 1, 0);
    // candidate sets of a round: W + candidate c, one row of W' tables per active candidate
    std::vector<otif_wsize> sets_mem((size_t)(m + 1) * 8);
    std::vector<const otif_wsize *> sets(m + 1);
    std::vector<int32_t> set_k(m + 1);
    std::vector<int> active;
    int nw = 1;
    // Σ est with W = {full frame}
    sets[0] = W;
    set_k[0] = 1;
    st = launch_select_multi(masks, n, gh, gw, g, sets.data(), set_k.data(), 1, wtab, sums, stream);
    if (st != OTIF_OK) return st;
    OTIF_CUDA(cudaMemcpyAsync(h.data(), sums, 8, cudaMemcpyDeviceToHost, stream));
    OTIF_CUDA(cudaStreamSynchronize(stream));
    chosen_idx[0] = -1;
    est[0] = n > 0 ? (int64_t)h[0] : 0;
    int64_t cur = est[0];
    while (nw < k) {
        active.clear();
        for (int c = 0; c < m; c++) {
            if (used[c]) continue;
            otif_wsize *set = &sets_mem[(size_t)active.size() * 8];
            for (int i = 0; i < nw; i++) set[i] = W[i];
            set[nw] = candidates[c];
            sets[active.size()] = set;
            set_k[active.size()] = nw + 1;
            active.push_back(c);
        }
        if (active.empty()) break;
        st = launch_select_multi(masks, n, gh, gw, g, sets.data(), set_k.data(), (int)active.size(), wtab, sums,
                                 stream);
        if (st != OTIF_OK) return st;
        OTIF_CUDA(cudaMemcpyAsync(h.data(), sums, active.size() * 8, cudaMemcpyDeviceToHost, stream));
        OTIF_CUDA(cudaStreamSynchronize(stream));
        int best = -1;
        int64_t best_sum = cur;
        for (size_t a = 0; a < active.size(); a++) {
            const int64_t s = n > 0 ? (int64_t)h[a] : 0;
            if (s < best_sum) { best_sum = s; best = active[a]; }  // greatest decrease; ties: earliest candidate
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
