// select.cu — stages 3 + 4: cell threshold, connected components and the greedy
// window grouping (P:L131, P:L147 threshold "exceeds"; P:L149–151 grouping;
// P:L133 full-frame fallback; P:L155 full frame always in W).  The exact procedure
// and tie-breaks are DESIGN.md §3 readings R6–R11, R14, R15; all decisions use
// integer arithmetic (int64 costs), so the output is bit-exact by construction.
//
// K5 select_kernel: one CTA per frame.
//   threshold -> union-find connected components in shared memory (lock-free
//   atomicCAS linking of the larger root under the smaller, so every root is its
//   component's first cell in raster order) -> block scan for raster-ordered
//   component ids -> shared-memory atomic bounding boxes -> phase A (parallel
//   best-gain pair search, block argmax with lexicographic tie-break) / phase B
//   (parallel first-overlapping-pair search) -> placement, strict full-frame
//   fallback, rank sort by (y, x) -> per-frame scratch.
// K6 compact_kernel: exclusive scan of per-frame counts (frame_offset, total) and
//   compaction of the windows into the caller's array in (frame, y, x) order.
#include <string.h>

#include <algorithm>

#include "common.cuh"

namespace otif {

constexpr int kSelThreads = 256;
constexpr int kMaxSizes = 8;

struct SelectParams {
    const float *scores;
    const uint8_t *mask_in;
    float thr;
    int n, gh, gw, cell, fw, fh, conn;
    int k;                      // |W|
    int sw[kMaxSizes], sh[kMaxSizes];
    long long cost[kMaxSizes];  // W' order (sorted by cost, area, w, h)
    int orig[kMaxSizes];        // original index of each W' entry
    int full;                   // W' index of fit(full frame)
    uint8_t *mask_out;
    otif_window *tmp;           // [n][cap_f]
    int cap_f;
    int *counts;                // [n]
};

__device__ __forceinline__ int uf_find(volatile int *par, int x) {
    while (true) {
        int p = par[x];
        if (p == x) return x;
        int gp = par[p];
        if (gp != p) par[x] = gp;  // path halving; parents only ever decrease
        x = p;
    }
}

__device__ __forceinline__ void uf_union(int *par, int a, int b) {
    volatile int *vp = par;
    while (true) {
        a = uf_find(vp, a);
        b = uf_find(vp, b);
        if (a == b) return;
        if (a < b) { int t = a; a = b; b = t; }   // link the larger root under the smaller
        int old = atomicCAS(&par[a], a, b);
        if (old == a) return;
        a = old;
    }
}

// fit: first W' entry containing a (w x h) rectangle
__device__ __forceinline__ int fit_size(const SelectParams &p, int w, int h) {
    for (int s = 0; s < p.k; s++)
        if (p.sw[s] >= w && p.sh[s] >= h) return s;
    return p.k - 1;  // unreachable: the full frame is in W and contains every cluster
}

struct Rect16 { short x0, y0, x1, y1; };  // cell units, half-open

__device__ __forceinline__ void rect_px(const SelectParams &p, Rect16 r, int &x0, int &y0, int &x1, int &y1) {
    x0 = r.x0 * p.cell;
    y0 = r.y0 * p.cell;
    x1 = min((int)r.x1 * p.cell, p.fw);
    y1 = min((int)r.y1 * p.cell, p.fh);
}

__device__ __forceinline__ int fit_rect(const SelectParams &p, Rect16 r) {
    int x0, y0, x1, y1;
    rect_px(p, r, x0, y0, x1, y1);
    return fit_size(p, x1 - x0, y1 - y0);
}

__device__ __forceinline__ Rect16 runion(Rect16 a, Rect16 b) {
    Rect16 u;
    u.x0 = min(a.x0, b.x0); u.y0 = min(a.y0, b.y0);
    u.x1 = max(a.x1, b.x1); u.y1 = max(a.y1, b.y1);
    return u;
}

__device__ __forceinline__ void place(const SelectParams &p, Rect16 r, int s, int &x, int &y) {
    int x0, y0, x1, y1;
    rect_px(p, r, x0, y0, x1, y1);
    x = min(max(x0 - (p.sw[s] - (x1 - x0)) / 2, 0), p.fw - p.sw[s]);
    y = min(max(y0 - (p.sh[s] - (y1 - y0)) / 2, 0), p.fh - p.sh[s]);
}

// block reduce of (gain desc, pair asc)
__device__ void block_argmax(long long &g, int &pp, long long *sg, int *sp) {
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        long long og = __shfl_down_sync(0xffffffffu, g, o);
        int op = __shfl_down_sync(0xffffffffu, pp, o);
        if (og > g || (og == g && op < pp)) { g = og; pp = op; }
    }
    if (lane == 0) { sg[warp] = g; sp[warp] = pp; }
    __syncthreads();
    if (warp == 0) {
        const int nw = blockDim.x >> 5;
        g = lane < nw ? sg[lane] : 0;
        pp = lane < nw ? sp[lane] : 0x7FFFFFFF;
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) {
            long long og = __shfl_down_sync(0xffffffffu, g, o);
            int op = __shfl_down_sync(0xffffffffu, pp, o);
            if (og > g || (og == g && op < pp)) { g = og; pp = op; }
        }
        if (lane == 0) { sg[0] = g; sp[0] = pp; }
    }
    __syncthreads();
    g = sg[0];
    pp = sp[0];
    __syncthreads();
}

__global__ void __launch_bounds__(kSelThreads) select_kernel(const __grid_constant__ SelectParams p) {
    extern __shared__ __align__(16) uint8_t smem[];
    const int cells = p.gh * p.gw;
    const int f = blockIdx.x;
    int *par = reinterpret_cast<int *>(smem);                             // [cells]
    short *cid = reinterpret_cast<short *>(par + cells);                  // [cells]
    uint8_t *cl_base = smem + ((cells * 6 + 15) & ~15);
    Rect16 *cl = reinterpret_cast<Rect16 *>(cl_base);                     // [cap]
    long long *cost = reinterpret_cast<long long *>(cl + p.cap_f);        // [cap]
    int *px = reinterpret_cast<int *>(cost + p.cap_f);                    // [cap]
    int *py = px + p.cap_f;                                               // [cap]
    signed char *sidx = reinterpret_cast<signed char *>(py + p.cap_f);    // [cap]
    signed char *alive = sidx + p.cap_f;                                  // [cap]
    __shared__ long long s_red_g[32];
    __shared__ int s_red_p[32];
    __shared__ int s_scan[kSelThreads];
    __shared__ int s_ncomp, s_min_pair;

    // --- stage 3: threshold (strict ">") ---
    for (int i = threadIdx.x; i < cells; i += blockDim.x) {
        bool m;
        if (p.mask_in) m = p.mask_in[(size_t)f * cells + i] != 0;
        else m = p.scores[(size_t)f * cells + i] > p.thr;
        par[i] = m ? i : -1;
        if (p.mask_out) p.mask_out[(size_t)f * cells + i] = m ? 1 : 0;
    }
    __syncthreads();

    // --- connected components, 4- or 8-connectivity (reading R6) ---
    for (int i = threadIdx.x; i < cells; i += blockDim.x) {
        if (par[i] < 0) continue;
        int y = i / p.gw, x = i - y * p.gw;
        if (x + 1 < p.gw && par[i + 1] >= 0) uf_union(par, i, i + 1);
        if (y + 1 < p.gh) {
            int d = i + p.gw;
            if (par[d] >= 0) uf_union(par, i, d);
            if (p.conn == 8) {
                if (x > 0 && par[d - 1] >= 0) uf_union(par, i, d - 1);
                if (x + 1 < p.gw && par[d + 1] >= 0) uf_union(par, i, d + 1);
            }
        }
    }
    __syncthreads();
    // flatten: resolve every root with read-only walks into a scratch array first (a
    // path-halving write racing with another thread's flatten store could leave a
    // non-root parent behind), then publish.  px/py (2*cap >= cells ints) are free here.
    {
        int *lab = px;
        for (int i = threadIdx.x; i < cells; i += blockDim.x) {
            int x = par[i];
            if (x >= 0)
                while (par[x] != x) x = par[x];
            lab[i] = x;
        }
        __syncthreads();
        for (int i = threadIdx.x; i < cells; i += blockDim.x) par[i] = lab[i];
    }
    __syncthreads();

    // raster-ordered component ids: exclusive scan of root flags over contiguous segments
    {
        const int seg = (cells + blockDim.x - 1) / blockDim.x;
        const int a = threadIdx.x * seg, b = min(a + seg, cells);
        int cnt = 0;
        for (int i = a; i < b; i++) cnt += (par[i] == i);
        s_scan[threadIdx.x] = cnt;
        __syncthreads();
        if (threadIdx.x == 0) {
            int run = 0;
            for (int t = 0; t < (int)blockDim.x; t++) { int v = s_scan[t]; s_scan[t] = run; run += v; }
            s_ncomp = run;
        }
        __syncthreads();
        int id = s_scan[threadIdx.x];
        for (int i = a; i < b; i++)
            if (par[i] == i) cid[i] = (short)id++;
    }
    __syncthreads();
    const int n = s_ncomp;
    if (n == 0) {
        if (threadIdx.x == 0) p.counts[f] = 0;
        return;
    }
    for (int c = threadIdx.x; c < n; c += blockDim.x) {
        cl[c].x0 = 0x7FFF; cl[c].y0 = 0x7FFF; cl[c].x1 = -1; cl[c].y1 = -1;
        alive[c] = 1;
    }
    __syncthreads();
    // bounding boxes in cell units: 32-bit shared atomics on shadow arrays carved from
    // px / py / cost (not yet in use)
    int *bx0 = px, *by0 = py;
    int *bx1 = reinterpret_cast<int *>(cost), *by1 = bx1 + p.cap_f;
    for (int c = threadIdx.x; c < n; c += blockDim.x) {
        bx0[c] = 0x7FFFFFFF; by0[c] = 0x7FFFFFFF; bx1[c] = -1; by1[c] = -1;
    }
    __syncthreads();
    for (int i = threadIdx.x; i < cells; i += blockDim.x) {
        if (par[i] < 0) continue;
        int c = cid[par[i]];
        int y = i / p.gw, x = i - y * p.gw;
        atomicMin(&bx0[c], x); atomicMin(&by0[c], y);
        atomicMax(&bx1[c], x + 1); atomicMax(&by1[c], y + 1);
    }
    __syncthreads();
    for (int c = threadIdx.x; c < n; c += blockDim.x) {
        Rect16 r;
        r.x0 = (short)bx0[c]; r.y0 = (short)by0[c]; r.x1 = (short)bx1[c]; r.y1 = (short)by1[c];
        cl[c] = r;
    }
    __syncthreads();
    for (int c = threadIdx.x; c < n; c += blockDim.x) {
        int s = fit_rect(p, cl[c]);
        sidx[c] = (signed char)s;
        cost[c] = p.cost[s];
    }
    __syncthreads();

    // --- grouping: phase A greedy merge, phase B disjointness (readings R7, R10) ---
    const long long npairs = (long long)n * n;
    while (true) {
        while (true) {  // phase A
            long long best = 0;
            int bp = 0x7FFFFFFF;
            for (long long q = threadIdx.x; q < npairs; q += blockDim.x) {
                int i = (int)(q / n), j = (int)(q - (long long)i * n);
                if (j <= i || !alive[i] || !alive[j]) continue;
                Rect16 u = runion(cl[i], cl[j]);
                long long g = cost[i] + cost[j] - p.cost[fit_rect(p, u)];
                if (g > best) { best = g; bp = (int)q; }   // q ascending per thread: first max is smallest
            }
            block_argmax(best, bp, s_red_g, s_red_p);
            if (best <= 0) break;                           // "merging offers no further improvement"
            if (threadIdx.x == 0) {
                int i = bp / n, j = bp - i * n;
                cl[i] = runion(cl[i], cl[j]);
                int s = fit_rect(p, cl[i]);
                sidx[i] = (signed char)s;
                cost[i] = p.cost[s];
                alive[j] = 0;
            }
            __syncthreads();
        }
        // phase B: place every cluster, merge the lexicographically first overlapping pair
        for (int c = threadIdx.x; c < n; c += blockDim.x)
            if (alive[c]) place(p, cl[c], sidx[c], px[c], py[c]);
        if (threadIdx.x == 0) s_min_pair = 0x7FFFFFFF;
        __syncthreads();
        for (long long q = threadIdx.x; q < npairs; q += blockDim.x) {
            int i = (int)(q / n), j = (int)(q - (long long)i * n);
            if (j <= i || !alive[i] || !alive[j]) continue;
            int si = sidx[i], sj = sidx[j];
            bool ox = px[i] < px[j] + p.sw[sj] && px[j] < px[i] + p.sw[si];
            bool oy = py[i] < py[j] + p.sh[sj] && py[j] < py[i] + p.sh[si];
            if (ox && oy) { atomicMin(&s_min_pair, (int)q); break; }  // later q of this thread are larger
        }
        __syncthreads();
        const int mp = s_min_pair;
        if (mp == 0x7FFFFFFF) break;
        if (threadIdx.x == 0) {
            int i = mp / n, j = mp - i * n;
            cl[i] = runion(cl[i], cl[j]);
            int s = fit_rect(p, cl[i]);
            sidx[i] = (signed char)s;
            cost[i] = p.cost[s];
            alive[j] = 0;
        }
        __syncthreads();
    }

    // --- emission: est(R), strict full-frame fallback (R11), (y, x) order (R15) ---
    long long est = 0;
    int m = 0;
    for (int c = threadIdx.x; c < n; c += blockDim.x)
        if (alive[c]) { est += cost[c]; m++; }
    {
        // block sums via the argmax scratch (sum reduction)
        const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
        for (int o = 16; o > 0; o >>= 1) {
            est += __shfl_down_sync(0xffffffffu, est, o);
            m += __shfl_down_sync(0xffffffffu, m, o);
        }
        if (lane == 0) { s_red_g[warp] = est; s_red_p[warp] = m; }
        __syncthreads();
        if (threadIdx.x == 0) {
            long long e = 0;
            int mm = 0;
            for (int w = 0; w < (int)(blockDim.x >> 5); w++) { e += s_red_g[w]; mm += s_red_p[w]; }
            s_red_g[0] = e;
            s_red_p[0] = mm;
        }
        __syncthreads();
        est = s_red_g[0];
        m = s_red_p[0];
    }
    otif_window *out = p.tmp + (size_t)f * p.cap_f;
    if (est > p.cost[p.full]) {
        if (threadIdx.x == 0) {
            otif_window w;
            w.frame = f; w.x = 0; w.y = 0; w.w = p.fw; w.h = p.fh; w.size_idx = p.orig[p.full];
            out[0] = w;
            p.counts[f] = 1;
        }
        return;
    }
    for (int c = threadIdx.x; c < n; c += blockDim.x) {
        if (!alive[c]) continue;
        int rank = 0;
        for (int d = 0; d < n; d++)
            if (alive[d] && (py[d] < py[c] || (py[d] == py[c] && px[d] < px[c]))) rank++;
        otif_window w;
        w.frame = f; w.x = px[c]; w.y = py[c];
        w.w = p.sw[sidx[c]]; w.h = p.sh[sidx[c]]; w.size_idx = p.orig[sidx[c]];
        out[rank] = w;
    }
    if (threadIdx.x == 0) p.counts[f] = m;
}

// K6: scan of per-frame counts + compaction into (frame, y, x) order
__global__ void __launch_bounds__(1024) compact_kernel(const otif_window *__restrict__ tmp, int cap_f,
                                                       const int *__restrict__ counts, int n, otif_window *out,
                                                       int capacity, int *frame_count, int *frame_offset, int *total) {
    __shared__ int s_warp[32];
    __shared__ int s_base;
    const int f0 = blockIdx.x * blockDim.x;
    // base = sum of counts of all earlier frames
    int part = 0;
    for (int i = threadIdx.x; i < f0; i += blockDim.x) part += counts[i];
    for (int o = 16; o > 0; o >>= 1) part += __shfl_down_sync(0xffffffffu, part, o);
    if ((threadIdx.x & 31) == 0) s_warp[threadIdx.x >> 5] = part;
    __syncthreads();
    if (threadIdx.x == 0) {
        int b = 0;
        for (int w = 0; w < (int)(blockDim.x >> 5); w++) b += s_warp[w];
        s_base = b;
    }
    __syncthreads();
    const int f = f0 + threadIdx.x;
    const int c = f < n ? counts[f] : 0;
    // block exclusive scan of c
    int v = c;
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    for (int o = 1; o < 32; o <<= 1) {
        int t = __shfl_up_sync(0xffffffffu, v, o);
        if (lane >= o) v += t;
    }
    __syncthreads();
    if (lane == 31) s_warp[warp] = v;
    __syncthreads();
    if (warp == 0) {
        int w = lane < (int)(blockDim.x >> 5) ? s_warp[lane] : 0;
        for (int o = 1; o < 32; o <<= 1) {
            int t = __shfl_up_sync(0xffffffffu, w, o);
            if (lane >= o) w += t;
        }
        s_warp[lane] = w;
    }
    __syncthreads();
    const int incl = v + (warp > 0 ? s_warp[warp - 1] : 0);
    const int off = s_base + incl - c;
    if (f < n) {
        frame_count[f] = c;
        frame_offset[f] = off;
        for (int i = 0; i < c; i++)
            if (off + i < capacity) out[off + i] = tmp[(size_t)f * cap_f + i];
        if (f == n - 1) *total = off + c;
    }
}

}  // namespace otif

using namespace otif;

static int sel_cap(int gh, int gw) { return (gh * gw + 1) / 2 > 1 ? (gh * gw + 1) / 2 : 1; }

static size_t sel_smem(int gh, int gw) {
    int cells = gh * gw, cap = sel_cap(gh, gw);
    size_t head = (size_t)round_up((int64_t)cells * 6, 16);
    return head + (size_t)cap * (8 + 8 + 4 + 4 + 1 + 1) + 64;
}

extern "C" size_t otif_select_workspace_bytes(int32_t n, int32_t gh, int32_t gw) {
    if (n < 0 || gh <= 0 || gw <= 0) return 0;
    return (size_t)round_up((int64_t)n * sel_cap(gh, gw) * sizeof(otif_window), 256) + (size_t)round_up((int64_t)n * 4, 256);
}

extern "C" otif_status otif_select_windows(const float *scores, const uint8_t *mask_in, float threshold, int32_t n,
                                           int32_t gh, int32_t gw, const otif_grid_desc *g, const otif_wsize *sizes,
                                           int32_t k, uint8_t *mask_out, otif_window *windows, int32_t capacity,
                                           int32_t *frame_count, int32_t *frame_offset, int32_t *total,
                                           void *workspace, size_t ws_bytes, cudaStream_t stream) {
    OTIF_REQUIRE(g && sizes, "otif_select_windows: NULL descriptor or sizes");
    OTIF_REQUIRE(n >= 0 && gh > 0 && gw > 0, "otif_select_windows: bad n/grid (%d, %dx%d)", n, gw, gh);
    OTIF_REQUIRE(g->frame_w > 0 && g->frame_h > 0 && g->cell > 0, "otif_select_windows: bad frame/cell");
    OTIF_REQUIRE(gh == (g->frame_h + g->cell - 1) / g->cell && gw == (g->frame_w + g->cell - 1) / g->cell,
                 "otif_select_windows: grid %dx%d != ceil(frame/cell) for %dx%d / %d", gw, gh, g->frame_w,
                 g->frame_h, g->cell);
    OTIF_REQUIRE((scores != nullptr) != (mask_in != nullptr), "otif_select_windows: exactly one of scores/mask_in");
    OTIF_REQUIRE(g->connectivity == 4 || g->connectivity == 8, "otif_select_windows: connectivity must be 4 or 8");
    OTIF_REQUIRE(k >= 1 && k <= kMaxSizes, "otif_select_windows: k=%d not in [1,8]", k);
    OTIF_REQUIRE(capacity >= 0, "otif_select_windows: negative capacity");
    OTIF_REQUIRE(gh * gw <= 8192, "otif_select_windows: grid of %d cells exceeds 8192", gh * gw);
    OTIF_REQUIRE(g->frame_w <= 0x7FFF && g->frame_h <= 0x7FFF && gw < 0x7FFF && gh < 0x7FFF,
                 "otif_select_windows: frame too large");
    bool full = false;
    for (int i = 0; i < k; i++) {
        OTIF_REQUIRE(sizes[i].w > 0 && sizes[i].h > 0 && sizes[i].w <= g->frame_w && sizes[i].h <= g->frame_h,
                     "otif_select_windows: size %d (%dx%d) not inside the %dx%d frame", i, sizes[i].w, sizes[i].h,
                     g->frame_w, g->frame_h);
        if (sizes[i].w == g->frame_w && sizes[i].h == g->frame_h) full = true;
    }
    OTIF_REQUIRE(full, "otif_select_windows: W must contain the full frame %dx%d (P:L155)", g->frame_w, g->frame_h);
    if (n == 0) {
        if (total) OTIF_CUDA(cudaMemsetAsync(total, 0, 4, stream));
        return OTIF_OK;
    }
    OTIF_REQUIRE(windows || capacity == 0, "otif_select_windows: NULL windows");
    OTIF_REQUIRE(frame_count && frame_offset && total && workspace, "otif_select_windows: NULL output");
    OTIF_REQUIRE(ws_bytes >= otif_select_workspace_bytes(n, gh, gw), "otif_select_windows: workspace too small");
    otif_status st = check_device(nullptr);
    if (st != OTIF_OK) return st;

    SelectParams p;
    memset(&p, 0, sizeof(p));
    p.scores = scores; p.mask_in = mask_in; p.thr = threshold;
    p.n = n; p.gh = gh; p.gw = gw; p.cell = g->cell; p.fw = g->frame_w; p.fh = g->frame_h;
    p.conn = g->connectivity; p.k = k;
    // W' = W sorted by (cost, w*h, w, h)
    int order[kMaxSizes];
    for (int i = 0; i < k; i++) order[i] = i;
    std::stable_sort(order, order + k, [&](int a, int b) {
        const otif_wsize &x = sizes[a], &y = sizes[b];
        if (x.cost != y.cost) return x.cost < y.cost;
        long long ax = (long long)x.w * x.h, ay = (long long)y.w * y.h;
        if (ax != ay) return ax < ay;
        if (x.w != y.w) return x.w < y.w;
        return x.h < y.h;
    });
    p.full = -1;
    for (int s = 0; s < k; s++) {
        const otif_wsize &z = sizes[order[s]];
        p.sw[s] = z.w; p.sh[s] = z.h; p.cost[s] = z.cost; p.orig[s] = order[s];
        if (p.full < 0 && z.w >= g->frame_w && z.h >= g->frame_h) p.full = s;
    }
    p.mask_out = mask_out;
    p.cap_f = sel_cap(gh, gw);
    uint8_t *ws = (uint8_t *)workspace;
    p.tmp = (otif_window *)ws;
    p.counts = (int *)(ws + round_up((int64_t)n * p.cap_f * sizeof(otif_window), 256));
    size_t smem = sel_smem(gh, gw);
    OTIF_CUDA(cudaFuncSetAttribute(select_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    select_kernel<<<n, kSelThreads, smem, stream>>>(p);
    OTIF_LAUNCH_CHECK();
    compact_kernel<<<(unsigned)cdiv(n, 1024), 1024, 0, stream>>>(p.tmp, p.cap_f, p.counts, n, windows, capacity,
                                                                 frame_count, frame_offset, total);
    OTIF_LAUNCH_CHECK();
    return OTIF_OK;
}
