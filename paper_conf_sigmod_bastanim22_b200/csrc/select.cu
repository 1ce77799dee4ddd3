// select.cu — stages 3 + 4: cell threshold, connected components and the greedy
// window grouping (P:L131, P:L147 threshold "exceeds"; P:L149–151 grouping;
// P:L133 full-frame fallback; P:L155 full frame always in W).  The exact procedure
// and tie-breaks are DESIGN.md §3 readings R6–R11, R14, R15; all decisions use
// integer arithmetic (int64 costs), so the output is bit-exact by construction.
//
// K5 select_kernel: ONE WARP PER FRAME (several frames per CTA, each warp owns a
// private shared-memory slice; warp-synchronous, no block barriers):
//   threshold (vectorised score loads) -> union-find connected components in shared
//   memory (lock-free atomicCAS linking of the larger root under the smaller, so a
//   root is its component's first cell in raster order) -> read-only flatten ->
//   warp scan for raster-ordered component ids -> shared atomic bounding boxes ->
//   phase A with a per-cluster best-partner cache (bg[i], bj[i] = best gain / partner
//   over j > i) over a one-byte fit-index matrix U[i][j] (n <= 128; a merge refreshes
//   row/column I and recomputes only the rows whose cached best can have changed —
//   larger n falls back to row rescans without the matrix) -> phase B (first
//   overlapping pair) ->
//   placement, strict full-frame fallback, rank sort by (y, x) -> per-frame scratch.
//   Optionally (pipeline) accumulates the run counters with a few atomics per frame.
// K6 compact_kernel: exclusive scan of per-frame counts (frame_offset, total) and
//   compaction of the windows into the caller's array in (frame, y, x) order.
#include <string.h>

#include <algorithm>
#include <vector>

#include "common.cuh"

namespace otif {

#ifdef OTIF_SEL_PROF     // profiling build: keep the grouping phases out of line (per-line ncu attribution)
#define OTIF_SEL_NOINLINE __noinline__
#else
#define OTIF_SEL_NOINLINE
#endif

constexpr int kSelWarpsMax = 16;
constexpr int kMatMax = 128;  // fit-matrix capacity (components per frame); larger n -> rescan path
constexpr int kSmallClusters = 64;  // components per frame in the first (high-occupancy) pass
constexpr int kMaxSizes = 8;

// One window-size set W' (sorted by (cost, w*h, w, h)) for the multi-candidate launch
// of NEXT-1 (blockIdx.y selects the table).
struct WTable {
    int k, full;
    int sw[8], sh[8], orig[8];
    long long cost[8];
};
static_assert(sizeof(WTable) <= 192, "tuning.cu sizes the W' table scratch at 192 B per entry");

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
    int frame_bytes;            // shared bytes per warp (frame slice)
    int nmat;                   // gain-matrix capacity (components); 0 = rescan path only
    int gmat_offset;            // byte offset of the gain matrix in a frame slice
    // pipeline-only (internal): run counters, global frame index base
    unsigned long long *ctr;
    int frame_base;
    unsigned long long *est_sum;  // internal: Σ est(R_t) over frames (window-size selection)
    unsigned long long *frame_hash;  // internal (pipeline): per-frame window hash [n] (the ctr[4] terms)
    // two-pass scheduling: pass 1 gives every frame a small slice (ccap clusters) and
    // defers frames with more components to pass 2 (full-size slices, frames from the list)
    int ccap;                   // cluster capacity of a slice
    int *defer_list;
    int *defer_count;
    int from_list;
    // NEXT-1 multi-candidate mode (select_kernel<true>): W' per blockIdx.y, est_sum[blockIdx.y],
    // no window / count outputs
    const WTable *wtab;
};

struct Rect16 { short x0, y0, x1, y1; };  // cell units, half-open

__device__ __forceinline__ void rect_px(const SelectParams &p, Rect16 r, int &x0, int &y0, int &x1, int &y1) {
    x0 = r.x0 * p.cell;
    y0 = r.y0 * p.cell;
    x1 = min((int)r.x1 * p.cell, p.fw);
    y1 = min((int)r.y1 * p.cell, p.fh);
}

// fit: first W' entry containing the cluster's pixel rectangle
__device__ __forceinline__ int fit_rect(const SelectParams &p, Rect16 r) {
    int x0, y0, x1, y1;
    rect_px(p, r, x0, y0, x1, y1);
    const int w = x1 - x0, h = y1 - y0;
    for (int s = 0; s < p.k; s++)
        if (p.sw[s] >= w && p.sh[s] >= h) return s;
    return p.full;  // unreachable: the full frame is in W and contains every cluster
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

__device__ __forceinline__ int uf_find(volatile int *par, int x) {
    while (true) {
        int q = par[x];
        if (q == x) return x;
        int g = par[q];
        // path halving; parents only ever decrease and always stay ancestors, so the
        // unsynchronised halving writes racing with other lanes' reads are benign
        // (compute-sanitizer racecheck reports them as warnings by design)
        if (g != q) par[x] = g;
        x = q;
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

__device__ __forceinline__ unsigned long long mix64(unsigned long long z) {
    z += 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}

constexpr long long kNoGain = (long long)0x8000000000000000ull;

struct Frame {  // one warp's shared-memory slice
    int *par;          // [cells]
    short *cid;        // [cells]
    Rect16 *cl;        // [cap]
    long long *cost;   // [cap]
    long long *bg;     // [cap] best gain over alive j > i
    short *bj;         // [cap] best partner
    signed char *sidx; // [cap]
    signed char *alive;// [cap]
    Rect16 *pw;        // [cap] placed windows (pixels) during a phase-B search; aliases par
};

// Phase B (reading R10): the lexicographically first pair (i < j) of alive clusters whose
// placed windows overlap.  The placements are computed once per search into F.pw (the
// union-find array, dead after the bounding boxes), then the warp tests 32 partners j of
// one i per step (ballot: the smallest j of the first i with an overlap).
__device__ __forceinline__ bool first_overlap(const SelectParams &p, Frame &F, int n, int lane, int &mi, int &mj) {
    for (int i = lane; i < n; i += 32) {
        if (!F.alive[i]) continue;
        int x, y;
        const int s = F.sidx[i];
        place(p, F.cl[i], s, x, y);
        Rect16 r;
        r.x0 = (short)x; r.y0 = (short)y; r.x1 = (short)(x + p.sw[s]); r.y1 = (short)(y + p.sh[s]);
        F.pw[i] = r;
    }
    __syncwarp();
    for (int i = 0; i + 1 < n; i++) {
        if (!F.alive[i]) continue;
        const Rect16 a = F.pw[i];
        for (int j0 = i + 1; j0 < n; j0 += 32) {
            const int j = j0 + lane;
            bool ov = false;
            if (j < n && F.alive[j]) {
                const Rect16 b = F.pw[j];
                ov = a.x0 < b.x1 && b.x0 < a.x1 && a.y0 < b.y1 && b.y0 < a.y1;
            }
            const unsigned m = __ballot_sync(0xffffffffu, ov);
            if (m) {
                mi = i;
                mj = j0 + __ffs(m) - 1;
                return true;
            }
        }
    }
    return false;
}

// best partner of row i over alive j > i (max gain, smallest j)
__device__ __forceinline__ void rescan_row(const SelectParams &p, Frame &F, int n, int i) {
    long long best = kNoGain;
    int bjv = -1;
    const Rect16 ri = F.cl[i];
    const long long ci = F.cost[i];
    for (int j = i + 1; j < n; j++) {
        if (!F.alive[j]) continue;
        long long g = ci + F.cost[j] - p.cost[fit_rect(p, runion(ri, F.cl[j]))];
        if (g > best) { best = g; bjv = j; }
    }
    F.bg[i] = best;
    F.bj[i] = (short)bjv;
}

// Greedy grouping with a pairwise fit matrix (n <= nmat).  U[i][j] (i < j, one byte)
// caches the W' index of fit(union(c_i, c_j)) — the gain is then cost_i + cost_j -
// cost[U[i][j]] (integer, exact) — and 0xFF marks a dead column.  Row bests (bg[i],
// bj[i]) = max gain over alive j > i, smallest j.  A merge of (I, J) refreshes the n
// entries of row/column I, kills column J, and recomputes only the affected row bests
// (row I and rows whose best was I or J, each by the whole warp over the cached row;
// rows i < I compare against their new U[i][I]) — O(n) work per merge on a warp.
// Same decisions as the oracle: max gain, ties to the lexicographically smallest (i, j).
constexpr uint8_t kDead = 0xFF;

__device__ __forceinline__ long long gain_u(const SelectParams &p, const Frame &F, int i, int j, uint8_t u) {
    return F.cost[i] + F.cost[j] - p.cost[u];
}

// warp-cooperative recompute of row i's best partner (all lanes call with the same i)
__device__ __forceinline__ void row_best_warp(const SelectParams &p, Frame &F, const uint8_t *U, int S, int n, int i,
                                              int lane) {
    long long best = kNoGain;
    int arg = 0x7FFF;
    const uint8_t *row = U + (size_t)i * S;
    for (int j = i + 1 + lane; j < n; j += 32) {
        const uint8_t u = row[j];
        if (u == kDead) continue;
        const long long g = gain_u(p, F, i, j, u);
        if (g > best) { best = g; arg = j; }   // j ascending per lane: first max is smallest
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        long long ob = __shfl_xor_sync(0xffffffffu, best, o);
        int oa = __shfl_xor_sync(0xffffffffu, arg, o);
        if (ob > best || (ob == best && oa < arg)) { best = ob; arg = oa; }
    }
    if (lane == 0) {
        F.bg[i] = arg == 0x7FFF ? kNoGain : best;
        F.bj[i] = (short)(arg == 0x7FFF ? -1 : arg);
    }
}

__device__ OTIF_SEL_NOINLINE void merge_update_mat(const SelectParams &p, Frame &F, int n, int lane, uint8_t *U, int I, int J) {
    const int S = p.nmat;
    __syncwarp();
    if (lane == 0) {
        F.cl[I] = runion(F.cl[I], F.cl[J]);
        int s = fit_rect(p, F.cl[I]);
        F.sidx[I] = (signed char)s;
        F.cost[I] = p.cost[s];
        F.alive[J] = 0;
    }
    __syncwarp();
    const Rect16 rI = F.cl[I];
    for (int j = lane; j < n; j += 32) {
        if (j < J) U[(size_t)j * S + J] = kDead;  // column J dies
        if (j == I || !F.alive[j]) continue;
        const uint8_t u = (uint8_t)fit_rect(p, runion(rI, F.cl[j]));
        if (j < I) U[(size_t)j * S + I] = u;
        else U[(size_t)I * S + j] = u;
    }
    __syncwarp();
    // lane-owned rows: cheap updates in place, full recomputes flagged for the warp
    for (int t = 0; t * 32 < n; t++) {
        const int i = t * 32 + lane;
        bool redo = false;
        if (i < n && F.alive[i]) {
            const int b = F.bj[i];
            if (i == I) {
                redo = true;                       // row I's entries all changed
            } else if (b == I) {                   // (i < I) best partner grew
                const long long g = gain_u(p, F, i, I, U[(size_t)i * S + I]);
                if (g >= F.bg[i]) F.bg[i] = g;     // still the max, same (smallest) partner
                else redo = true;                  // decreased: another partner may win
            } else if (b == J) {                   // best partner died
                // if I (< J) now reaches the old best gain it is the new best: any other
                // partner with that gain has an index > J (J was the smallest such)
                const long long g = i < I ? gain_u(p, F, i, I, U[(size_t)i * S + I]) : kNoGain;
                if (i < I && g >= F.bg[i]) { F.bg[i] = g; F.bj[i] = (short)I; }
                else redo = true;
            } else if (i < I) {
                const uint8_t u = U[(size_t)i * S + I];
                const long long g = gain_u(p, F, i, I, u);
                if (g > F.bg[i] || (g == F.bg[i] && I < b)) { F.bg[i] = g; F.bj[i] = (short)I; }
            }
        }
        unsigned m = __ballot_sync(0xffffffffu, redo);
        __syncwarp();  // this group's bj/bg reads happen-before lane 0's rewrites below
        while (m) {
            const int l = __ffs(m) - 1;
            m &= m - 1;
            row_best_warp(p, F, U, S, n, t * 32 + l, lane);
        }
    }
    __syncwarp();
}

__device__ OTIF_SEL_NOINLINE bool greedy_matrix(const SelectParams &p, Frame &F, int n, int lane, uint8_t *U) {
    const int S = p.nmat;
    // fit matrix and row bests in one pass: row i's entries are computed by the lanes that
    // reduce them (all clusters alive; same max / smallest-j rule as row_best_warp)
    for (int i = 0; i < n; i++) {
        const Rect16 ri = F.cl[i];
        const long long ci = F.cost[i];
        long long best = kNoGain;
        int arg = 0x7FFF;
        for (int j = i + 1 + lane; j < n; j += 32) {
            const uint8_t u = (uint8_t)fit_rect(p, runion(ri, F.cl[j]));
            U[(size_t)i * S + j] = u;
            const long long g = ci + F.cost[j] - p.cost[u];
            if (g > best) { best = g; arg = j; }
        }
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) {
            long long ob = __shfl_xor_sync(0xffffffffu, best, o);
            int oa = __shfl_xor_sync(0xffffffffu, arg, o);
            if (ob > best || (ob == best && oa < arg)) { best = ob; arg = oa; }
        }
        if (lane == 0) {
            F.bg[i] = arg == 0x7FFF ? kNoGain : best;
            F.bj[i] = (short)(arg == 0x7FFF ? -1 : arg);
        }
    }
    __syncwarp();
    while (true) {
        while (true) {  // phase A
            long long Gv = kNoGain;
            int I = 0x7FFF;
            for (int i = lane; i < n; i += 32)
                if (F.alive[i] && (F.bg[i] > Gv || (F.bg[i] == Gv && i < I))) { Gv = F.bg[i]; I = i; }
#pragma unroll
            for (int o = 16; o > 0; o >>= 1) {
                long long og = __shfl_xor_sync(0xffffffffu, Gv, o);
                int oi = __shfl_xor_sync(0xffffffffu, I, o);
                if (og > Gv || (og == Gv && oi < I)) { Gv = og; I = oi; }
            }
            if (Gv <= 0) break;
            merge_update_mat(p, F, n, lane, U, I, F.bj[I]);
            if (F.sidx[I] == p.full) return true;  // exact full-frame exit (see select_kernel)
        }
        // phase B: lexicographically first pair of alive clusters whose placed windows overlap
        int mi, mj;
        if (!first_overlap(p, F, n, lane, mi, mj)) break;
        merge_update_mat(p, F, n, lane, U, mi, mj);
        if (F.sidx[mi] == p.full) return true;
    }
    return false;
}

// Greedy grouping without the fit matrix (n > nmat or costs too large for the matrix):
// row rescans.  Returns true on the exact full-frame exit (see select_kernel).
__device__ bool greedy_rescan(const SelectParams &p, Frame &F, int n, int lane) {
    while (true) {
        for (int i = lane; i < n; i += 32)
            if (F.alive[i]) rescan_row(p, F, n, i);
        __syncwarp();
        while (true) {  // phase A
            long long G = kNoGain;
            int I = 0x7FFF;
            for (int i = lane; i < n; i += 32)
                if (F.alive[i] && (F.bg[i] > G || (F.bg[i] == G && i < I))) { G = F.bg[i]; I = i; }
#pragma unroll
            for (int o = 16; o > 0; o >>= 1) {
                long long og = __shfl_xor_sync(0xffffffffu, G, o);
                int oi = __shfl_xor_sync(0xffffffffu, I, o);
                if (og > G || (og == G && oi < I)) { G = og; I = oi; }
            }
            if (G <= 0) break;  // "once merging offers no further improvement" (strict)
            const int J = F.bj[I];
            __syncwarp();
            if (lane == 0) {
                F.cl[I] = runion(F.cl[I], F.cl[J]);
                int s = fit_rect(p, F.cl[I]);
                F.sidx[I] = (signed char)s;
                F.cost[I] = p.cost[s];
                F.alive[J] = 0;
            }
            __syncwarp();
            if (F.sidx[I] == p.full) return true;
            for (int i = lane; i < n; i += 32) {
                if (!F.alive[i]) continue;
                const int b = F.bj[i];
                if (i == I || b == I || b == J) {
                    rescan_row(p, F, n, i);
                } else if (i < I) {
                    long long g = F.cost[i] + F.cost[I] - p.cost[fit_rect(p, runion(F.cl[i], F.cl[I]))];
                    if (g > F.bg[i] || (g == F.bg[i] && I < b)) { F.bg[i] = g; F.bj[i] = (short)I; }
                }
            }
            __syncwarp();
        }
        // phase B: merge the lexicographically first pair whose placed windows overlap
        int mi, mj;
        if (!first_overlap(p, F, n, lane, mi, mj)) break;
        __syncwarp();
        if (lane == 0) {
            F.cl[mi] = runion(F.cl[mi], F.cl[mj]);
            int s = fit_rect(p, F.cl[mi]);
            F.sidx[mi] = (signed char)s;
            F.cost[mi] = p.cost[s];
            F.alive[mj] = 0;
        }
        __syncwarp();
        if (F.sidx[mi] == p.full) return true;
    }
    return false;

}

// (MULTI returns after the est sum: the emission code below is unreachable there by design)
#pragma nv_diag_suppress 128
template <bool MULTI>
__global__ void __launch_bounds__(kSelWarpsMax * 32) select_kernel(const __grid_constant__ SelectParams pin) {
    extern __shared__ __align__(16) uint8_t smem[];
    // MULTI (NEXT-1): this CTA row groups its frames with the W' of candidate set blockIdx.y
    SelectParams loc;
    if constexpr (MULTI) {
        loc = pin;
        const WTable &t = pin.wtab[blockIdx.y];
        loc.k = t.k;
        loc.full = t.full;
        for (int s = 0; s < kMaxSizes; s++) {
            loc.sw[s] = t.sw[s]; loc.sh[s] = t.sh[s]; loc.orig[s] = t.orig[s]; loc.cost[s] = t.cost[s];
        }
        loc.est_sum = pin.est_sum + blockIdx.y;
    }
    const SelectParams &p = MULTI ? loc : pin;
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    int f = blockIdx.x * (blockDim.x >> 5) + wid;
    if (p.from_list) {
        if (f >= *p.defer_count) return;
        f = p.defer_list[f];
    } else if (f >= p.n) {
        return;
    }
    const int cells = p.gh * p.gw;
    const int cap = p.ccap;
    uint8_t *base = smem + (size_t)wid * p.frame_bytes;
    Frame F;
    F.par = reinterpret_cast<int *>(base);
    F.cid = reinterpret_cast<short *>(F.par + cells);
    uint8_t *cb = base + ((cells * 6 + 15) & ~15);
    F.cl = reinterpret_cast<Rect16 *>(cb);
    F.cost = reinterpret_cast<long long *>(F.cl + cap);
    F.bg = F.cost + cap;
    F.bj = reinterpret_cast<short *>(F.bg + cap);
    F.sidx = reinterpret_cast<signed char *>(F.bj + cap);
    F.alive = F.sidx + cap;
    F.pw = reinterpret_cast<Rect16 *>(base);   // par / cid are dead once the boxes are built

    // --- stage 3: threshold (strict ">") ---
    int npos = 0;
    for (int i = lane; i < cells; i += 32) {
        bool m;
        if (p.mask_in) m = p.mask_in[(size_t)f * cells + i] != 0;
        else m = __ldg(p.scores + (size_t)f * cells + i) > p.thr;
        F.par[i] = m ? i : -1;
        npos += m;
        if (p.mask_out) p.mask_out[(size_t)f * cells + i] = m ? 1 : 0;
    }
    __syncwarp();

    // --- connected components, 4- or 8-connectivity (reading R6) ---
    for (int i = lane; i < cells; i += 32) {
        if (F.par[i] < 0) continue;
        int y = i / p.gw, x = i - y * p.gw;
        if (x + 1 < p.gw && F.par[i + 1] >= 0) uf_union(F.par, i, i + 1);
        if (y + 1 < p.gh) {
            int d = i + p.gw;
            if (F.par[d] >= 0) uf_union(F.par, i, d);
            if (p.conn == 8) {
                if (x > 0 && F.par[d - 1] >= 0) uf_union(F.par, i, d - 1);
                if (x + 1 < p.gw && F.par[d + 1] >= 0) uf_union(F.par, i, d + 1);
            }
        }
    }
    __syncwarp();
    // read-only flatten into scratch (the cid array, free until the id scan), then publish
    {
        short *lab = F.cid;
        for (int i = lane; i < cells; i += 32) {
            int x = F.par[i];
            if (x >= 0)
                while (F.par[x] != x) x = F.par[x];
            lab[i] = (short)x;
        }
        __syncwarp();
        for (int i = lane; i < cells; i += 32) F.par[i] = lab[i];
        __syncwarp();
    }
    // raster-ordered component ids: warp exclusive scan of root flags over contiguous segments
    int n;
    {
        const int seg = (cells + 31) / 32;
        const int a = lane * seg, b = min(a + seg, cells);
        int cnt = 0;
        for (int i = a; i < b; i++) cnt += (F.par[i] == i);
        int incl = cnt;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            int t = __shfl_up_sync(0xffffffffu, incl, o);
            if (lane >= o) incl += t;
        }
        n = __shfl_sync(0xffffffffu, incl, 31);
        int id = incl - cnt;
        for (int i = a; i < b; i++)
            if (F.par[i] == i) F.cid[i] = (short)id++;
    }
    __syncwarp();
    for (int o = 16; o > 0; o >>= 1) npos += __shfl_xor_sync(0xffffffffu, npos, o);
    otif_window *out = p.tmp + (size_t)f * p.cap_f;
    if (n > cap) {  // more components than this slice holds: defer to the full-size pass
        if (lane == 0) p.defer_list[atomicAdd(p.defer_count, 1)] = f;
        return;
    }
    if (n == 0) {
        if (lane == 0 && !MULTI) {
            p.counts[f] = 0;
            if (p.ctr) atomicAdd(&p.ctr[0], 1ull);
            if (p.frame_hash) p.frame_hash[f] = 0ull;
        }
        return;
    }
    // bounding boxes (cell units) with 32-bit shared atomics on shadow arrays in bg (2*cap ints)
    // and cost (2*cap ints), both unused until the boxes are final
    {
        int *bx0 = reinterpret_cast<int *>(F.bg), *by0 = bx0 + cap;
        int *bx1 = reinterpret_cast<int *>(F.cost), *by1 = bx1 + cap;
        for (int c = lane; c < n; c += 32) {
            bx0[c] = 0x7FFFFFFF; by0[c] = 0x7FFFFFFF; bx1[c] = -1; by1[c] = -1;
        }
        __syncwarp();
        for (int i = lane; i < cells; i += 32) {
            if (F.par[i] < 0) continue;
            int c = F.cid[F.par[i]];
            int y = i / p.gw, x = i - y * p.gw;
            atomicMin(&bx0[c], x); atomicMin(&by0[c], y);
            atomicMax(&bx1[c], x + 1); atomicMax(&by1[c], y + 1);
        }
        __syncwarp();
        for (int c = lane; c < n; c += 32) {
            Rect16 r;
            r.x0 = (short)bx0[c]; r.y0 = (short)by0[c]; r.x1 = (short)bx1[c]; r.y1 = (short)by1[c];
            F.cl[c] = r;
        }
        __syncwarp();
        for (int c = lane; c < n; c += 32) {
            int s = fit_rect(p, F.cl[c]);
            F.sidx[c] = (signed char)s;
            F.cost[c] = p.cost[s];
            F.alive[c] = 1;
        }
        __syncwarp();
    }

    // --- grouping: phase A greedy merge, phase B disjointness (readings R7, R10) ---
    // Exact full-frame exit: once a cluster's fit is the full frame (W' index p.full), the
    // output is the single window (0, 0, Wd, Hd).  Its placement overlaps every other
    // window, so phase B merges every cluster into it; a union containing it still fits
    // p.full first (nothing cheaper contains the smaller rectangle); the final
    // est = T_full is not > T_full, so the result is exactly the fallback window below.
    bool full_hit = __any_sync(0xffffffffu, [&] {
        bool h = false;
        for (int c = lane; c < n; c += 32) h |= F.sidx[c] == p.full;
        return h;
    }());
    if (!full_hit) {
        if (p.nmat > 0 && n <= p.nmat) full_hit = greedy_matrix(p, F, n, lane, base + p.gmat_offset);
        else full_hit = greedy_rescan(p, F, n, lane);
    }

    // --- emission: est(R), strict full-frame fallback (R11), (y, x) order (R15) ---
    long long est = 0;
    int m = 0;
    for (int c = lane; c < n; c += 32)
        if (F.alive[c]) { est += F.cost[c]; m++; }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        est += __shfl_xor_sync(0xffffffffu, est, o);
        m += __shfl_xor_sync(0xffffffffu, m, o);
    }
    unsigned long long hsh = 0, pix = 0;
    if (full_hit || est > p.cost[p.full]) {
        if (MULTI) {
            if (lane == 0) atomicAdd(p.est_sum, (unsigned long long)p.cost[p.full]);
            return;
        }
        if (lane == 0) {
            otif_window w;
            w.frame = f; w.x = 0; w.y = 0; w.w = p.fw; w.h = p.fh; w.size_idx = p.orig[p.full];
            out[0] = w;
            p.counts[f] = 1;
            if (p.est_sum) atomicAdd(p.est_sum, (unsigned long long)p.cost[p.full]);
            if (p.ctr || p.frame_hash) {
                unsigned long long gf = (unsigned long long)(unsigned)(f + p.frame_base);
                const unsigned long long h = mix64((gf << 32) ^ mix64(((unsigned long long)p.fw << 20) ^
                                                                      ((unsigned long long)p.fh << 4) ^ (unsigned)w.size_idx));
                if (p.frame_hash) p.frame_hash[f] = h;
                if (p.ctr) {
                    atomicAdd(&p.ctr[0], 1ull);
                    atomicAdd(&p.ctr[1], (unsigned long long)npos);
                    atomicAdd(&p.ctr[2], 1ull);
                    atomicAdd(&p.ctr[3], (unsigned long long)p.fw * p.fh);
                    atomicAdd(&p.ctr[4], h);
                    atomicAdd(&p.ctr[5 + w.size_idx], 1ull);
                }
            }
        }
        return;
    }
    if constexpr (MULTI) {
        if (lane == 0) atomicAdd(p.est_sum, (unsigned long long)est);
        return;
    }
    // rank each alive cluster's placed window by (y, x); placements recomputed per lane
    for (int c = lane; c < n; c += 32) {
        if (!F.alive[c]) continue;
        int xc, yc, sc = F.sidx[c];
        place(p, F.cl[c], sc, xc, yc);
        int rank = 0;
        for (int d = 0; d < n; d++) {
            if (!F.alive[d] || d == c) continue;
            int xd, yd;
            place(p, F.cl[d], F.sidx[d], xd, yd);
            rank += (yd < yc || (yd == yc && xd < xc));
        }
        otif_window w;
        w.frame = f; w.x = xc; w.y = yc; w.w = p.sw[sc]; w.h = p.sh[sc]; w.size_idx = p.orig[sc];
        out[rank] = w;
        if (p.ctr || p.frame_hash) {
            unsigned long long gf = (unsigned long long)(unsigned)(f + p.frame_base);
            unsigned long long key = (gf << 32) ^ ((unsigned long long)(unsigned)xc << 16) ^ (unsigned)yc;
            hsh += mix64(key ^ mix64(((unsigned long long)w.w << 20) ^ ((unsigned long long)w.h << 4) ^
                                     (unsigned)w.size_idx));
            pix += (unsigned long long)w.w * w.h;
            if (p.ctr) atomicAdd(&p.ctr[5 + w.size_idx], 1ull);
        }
    }
    if (p.ctr || p.frame_hash) {
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) {
            hsh += __shfl_xor_sync(0xffffffffu, hsh, o);
            pix += __shfl_xor_sync(0xffffffffu, pix, o);
        }
    }
    if (lane == 0) {
        p.counts[f] = m;
        if (p.frame_hash) p.frame_hash[f] = hsh;
        if (p.est_sum) atomicAdd(p.est_sum, (unsigned long long)est);
        if (p.ctr) {
            atomicAdd(&p.ctr[0], 1ull);
            atomicAdd(&p.ctr[1], (unsigned long long)npos);
            atomicAdd(&p.ctr[2], (unsigned long long)m);
            atomicAdd(&p.ctr[3], pix);
            atomicAdd(&p.ctr[4], hsh);
        }
    }
}

#pragma nv_diag_default 128

// K6: scan of per-frame counts + compaction into (frame, y, x) order
__global__ void __launch_bounds__(1024) compact_kernel(const otif_window *__restrict__ tmp, int cap_f,
                                                       const int *__restrict__ counts, int n, otif_window *out,
                                                       int capacity, int *frame_count, int *frame_offset, int *total) {
    __shared__ int s_warp[32];
    __shared__ int s_base;
    const int f0 = blockIdx.x * blockDim.x;
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

static int sel_cap(int gh, int gw) { return (gh * gw + 1) / 2 > 1 ? (gh * gw + 1) / 2 : 1; }

// shared bytes of one frame slice holding ccap clusters and an nmat x nmat fit matrix
static int sel_frame_bytes(int gh, int gw, int ccap, int nmat, int *gmat_offset) {
    int cells = gh * gw;
    int head = (cells * 6 + 15) & ~15;
    // cl 8 + cost 8 + bg 8 + bj 2 + sidx 1 + alive 1 bytes per cluster
    int body = (int)round_up(head + (int64_t)ccap * 28, 16);
    *gmat_offset = body;
    return body + (int)round_up((int64_t)nmat * nmat, 16);
}

// W' = W sorted by (cost, w*h, w, h); full = first entry holding the whole frame
static void sort_sizes(const otif_wsize *sizes, int k, int fw, int fh, WTable &t) {
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
    memset(&t, 0, sizeof(t));
    t.k = k;
    t.full = -1;
    for (int s = 0; s < k; s++) {
        const otif_wsize &z = sizes[order[s]];
        t.sw[s] = z.w; t.sh[s] = z.h; t.cost[s] = z.cost; t.orig[s] = order[s];
        if (t.full < 0 && z.w >= fw && z.h >= fh) t.full = s;
    }
}

// internal entry: counters and global frame base for the pipeline (NULL / 0 from the ABI)
otif_status launch_select(const float *scores, const uint8_t *mask_in, float threshold, int32_t n, int32_t gh,
                          int32_t gw, const otif_grid_desc *g, const otif_wsize *sizes, int32_t k, uint8_t *mask_out,
                          otif_window *windows, int32_t capacity, int32_t *frame_count, int32_t *frame_offset,
                          int32_t *total, void *workspace, size_t ws_bytes, cudaStream_t stream,
                          unsigned long long *ctr, int frame_base, unsigned long long *est_sum,
                          unsigned long long *frame_hash) {
    SelectParams p;
    memset(&p, 0, sizeof(p));
    p.scores = scores; p.mask_in = mask_in; p.thr = threshold;
    p.n = n; p.gh = gh; p.gw = gw; p.cell = g->cell; p.fw = g->frame_w; p.fh = g->frame_h;
    p.conn = g->connectivity; p.k = k;
    // W' = W sorted by (cost, w*h, w, h)
    {
        WTable t;
        sort_sizes(sizes, k, g->frame_w, g->frame_h, t);
        p.full = t.full;
        for (int s = 0; s < k; s++) { p.sw[s] = t.sw[s]; p.sh[s] = t.sh[s]; p.cost[s] = t.cost[s]; p.orig[s] = t.orig[s]; }
    }
    p.mask_out = mask_out;
    p.cap_f = sel_cap(gh, gw);
    uint8_t *ws = (uint8_t *)workspace;
    p.tmp = (otif_window *)ws;
    p.counts = (int *)(ws + round_up((int64_t)n * p.cap_f * sizeof(otif_window), 256));
    // fit matrix only when int32 gains are exact
    long long max_cost = 0;
    for (int s = 0; s < k; s++) max_cost = sizes[s].cost > max_cost ? sizes[s].cost : max_cost;
    bool small_costs = max_cost < (1ll << 30);
    for (int s = 0; s < k; s++) small_costs = small_costs && sizes[s].cost >= 0;
    p.ctr = ctr;
    p.frame_base = frame_base;
    p.est_sum = est_sum;
    p.frame_hash = frame_hash;
    p.defer_list = p.counts + round_up(n, 64);
    p.defer_count = p.defer_list + round_up(n, 64);
    OTIF_CUDA(cudaMemsetAsync(p.defer_count, 0, 4, stream));
    int num_sms = 148;
    check_device(&num_sms);
    const size_t cap_bytes = 200 * 1024;
    // a batch that fits ONE wave with full-size slices takes a single pass with them (the
    // small-slice pass only buys occupancy, and a deferred frame redoes its components)
    int small_cap = p.cap_f < kSmallClusters ? p.cap_f : kSmallClusters;
    {
        int gm;
        const int fb = sel_frame_bytes(gh, gw, p.cap_f, small_costs ? (int)round_up(p.cap_f < kMatMax ? p.cap_f : kMatMax, 8) : 0, &gm);
        const int64_t full_warps = std::max<int64_t>(1, std::min<int64_t>(kSelWarpsMax, (int64_t)cap_bytes / fb));
        if ((int64_t)n <= full_warps * num_sms) small_cap = p.cap_f;
    }
    for (int pass = 0; pass < 2; pass++) {
        // pass 0: small slices (<= kSmallClusters components, many frames per SM);
        // pass 1: the deferred frames with full-size slices
        const int ccap = pass == 0 ? small_cap : p.cap_f;
        if (pass == 1 && ccap == small_cap) break;  // nothing deferred
        p.ccap = ccap;
        p.from_list = pass;
        p.nmat = small_costs ? (int)round_up(ccap < kMatMax ? ccap : kMatMax, 8) : 0;
        p.frame_bytes = sel_frame_bytes(gh, gw, ccap, p.nmat, &p.gmat_offset);
        int warps = (int)(cap_bytes / p.frame_bytes);
        warps = warps < 1 ? 1 : (warps > kSelWarpsMax ? kSelWarpsMax : warps);
        if (pass == 0) {  // spread small batches over the SMs rather than packing frames into few CTAs
            while (warps > 1 && cdiv(n, warps) < 2 * num_sms) warps--;
        }
        if (warps > n) warps = n;
        const size_t smem = (size_t)warps * p.frame_bytes;
        OTIF_CUDA(cudaFuncSetAttribute(select_kernel<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
        select_kernel<false><<<(unsigned)cdiv(n, warps), warps * 32, smem, stream>>>(p);
        OTIF_LAUNCH_CHECK();
    }
    compact_kernel<<<(unsigned)cdiv(n, 1024), 1024, 0, stream>>>(p.tmp, p.cap_f, p.counts, n, windows, capacity,
                                                                 frame_count, frame_offset, total);
    OTIF_LAUNCH_CHECK();
    return OTIF_OK;
}

// NEXT-1: Σ_t est(R(I_t; W_c)) for m window-size sets W_c (k_c <= 8 sizes each, host) over
// n masks in ONE launch (grid.y = m; full-size slices, no deferred pass) -> est_sums[m]
// (device, zeroed here).  wtab_dev: device scratch of m WTable entries.
otif_status launch_select_multi(const uint8_t *masks, int32_t n, int32_t gh, int32_t gw, const otif_grid_desc *g,
                                const otif_wsize *const *sets, const int32_t *set_k, int32_t m, void *wtab_dev,
                                unsigned long long *est_sums, cudaStream_t stream) {
    if (m <= 0) return OTIF_OK;
    OTIF_CUDA(cudaMemsetAsync(est_sums, 0, (size_t)m * 8, stream));
    if (n <= 0) return OTIF_OK;
    std::vector<WTable> tabs(m);
    long long max_cost = 0;
    bool nonneg = true;
    for (int c = 0; c < m; c++) {
        sort_sizes(sets[c], set_k[c], g->frame_w, g->frame_h, tabs[c]);
        for (int s = 0; s < set_k[c]; s++) {
            max_cost = sets[c][s].cost > max_cost ? sets[c][s].cost : max_cost;
            nonneg = nonneg && sets[c][s].cost >= 0;
        }
    }
    OTIF_CUDA(cudaMemcpyAsync(wtab_dev, tabs.data(), (size_t)m * sizeof(WTable), cudaMemcpyHostToDevice, stream));
    SelectParams p;
    memset(&p, 0, sizeof(p));
    p.mask_in = masks;
    p.n = n; p.gh = gh; p.gw = gw; p.cell = g->cell; p.fw = g->frame_w; p.fh = g->frame_h;
    p.conn = g->connectivity;
    p.cap_f = sel_cap(gh, gw);
    p.ccap = p.cap_f;
    p.nmat = (max_cost < (1ll << 30) && nonneg) ? (int)round_up(p.ccap < kMatMax ? p.ccap : kMatMax, 8) : 0;
    p.frame_bytes = sel_frame_bytes(gh, gw, p.ccap, p.nmat, &p.gmat_offset);
    p.wtab = reinterpret_cast<const WTable *>(wtab_dev);
    p.est_sum = est_sums;
    int warps = (int)((size_t)200 * 1024 / p.frame_bytes);
    warps = warps < 1 ? 1 : (warps > kSelWarpsMax ? kSelWarpsMax : warps);
    if (warps > n) warps = n;
    const size_t smem = (size_t)warps * p.frame_bytes;
    OTIF_REQUIRE(smem <= 227 * 1024, "otif_choose_window_sizes: grid of %d cells too large", gh * gw);
    OTIF_CUDA(cudaFuncSetAttribute(select_kernel<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    select_kernel<true><<<dim3((unsigned)cdiv(n, warps), (unsigned)m), warps * 32, smem, stream>>>(p);
    OTIF_LAUNCH_CHECK();
    return OTIF_OK;
}

size_t select_workspace_bytes(int32_t n, int32_t gh, int32_t gw) {
    if (n < 0 || gh <= 0 || gw <= 0) return 0;
    // per-frame window scratch; counts, the deferred-frame list and its counter
    return (size_t)round_up((int64_t)n * sel_cap(gh, gw) * sizeof(otif_window), 256) +
           (size_t)round_up((round_up(n, 64) * 2 + 64) * 4, 256);
}

otif_status validate_select(const float *scores, const uint8_t *mask_in, int32_t n, int32_t gh, int32_t gw,
                            const otif_grid_desc *g, const otif_wsize *sizes, int32_t k, int32_t capacity) {
    OTIF_REQUIRE(g && sizes, "otif_select_windows: NULL descriptor or sizes");
    OTIF_REQUIRE(n >= 0 && gh > 0 && gw > 0, "otif_select_windows: bad n/grid (%d, %dx%d)", n, gw, gh);
    OTIF_REQUIRE(g->frame_w > 0 && g->frame_h > 0 && g->cell > 0, "otif_select_windows: bad frame/cell");
    OTIF_REQUIRE(gh == (g->frame_h + g->cell - 1) / g->cell && gw == (g->frame_w + g->cell - 1) / g->cell,
                 "otif_select_windows: grid %dx%d != ceil(frame/cell) for %dx%d / %d", gw, gh, g->frame_w,
                 g->frame_h, g->cell);
    OTIF_REQUIRE(n == 0 || (scores != nullptr) != (mask_in != nullptr),
                 "otif_select_windows: exactly one of scores/mask_in");
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
    return OTIF_OK;
}

}  // namespace otif

using namespace otif;

extern "C" size_t otif_select_workspace_bytes(int32_t n, int32_t gh, int32_t gw) {
    return select_workspace_bytes(n, gh, gw);
}

extern "C" otif_status otif_select_windows(const float *scores, const uint8_t *mask_in, float threshold, int32_t n,
                                           int32_t gh, int32_t gw, const otif_grid_desc *g, const otif_wsize *sizes,
                                           int32_t k, uint8_t *mask_out, otif_window *windows, int32_t capacity,
                                           int32_t *frame_count, int32_t *frame_offset, int32_t *total,
                                           void *workspace, size_t ws_bytes, cudaStream_t stream,
                                           int64_t *est_sum) {
    otif_status st = validate_select(scores, mask_in, n, gh, gw, g, sizes, k, capacity);
    if (st != OTIF_OK) return st;
    if (est_sum) OTIF_CUDA(cudaMemsetAsync(est_sum, 0, 8, stream));
    if (n == 0) {
        if (total) OTIF_CUDA(cudaMemsetAsync(total, 0, 4, stream));
        return OTIF_OK;
    }
    OTIF_REQUIRE(windows || capacity == 0, "otif_select_windows: NULL windows");
    OTIF_REQUIRE(frame_count && frame_offset && total && workspace, "otif_select_windows: NULL output");
    OTIF_REQUIRE(ws_bytes >= otif_select_workspace_bytes(n, gh, gw), "otif_select_windows: workspace too small");
    st = check_device(nullptr);
    if (st != OTIF_OK) return st;
    return launch_select(scores, mask_in, threshold, n, gh, gw, g, sizes, k, mask_out, windows, capacity, frame_count,
                         frame_offset, total, workspace, ws_bytes, stream, nullptr, 0,
                         reinterpret_cast<unsigned long long *>(est_sum), nullptr);
}
