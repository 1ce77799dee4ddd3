// tracks.cu — §8(f) NEXT-4, track refinement on sm_100a.
//
//   resample_kernel  warp per track: arc-length resampling to N points (R21); the
//                    lanes compute segment lengths, the fp64 prefix runs in index order
//                    with one IEEE rounding per operation.
//   DBSCAN in a spatially sorted order of S* (sort_kernel: 16-bit start/end
//   cell keys, stable radix; gather_kernel: sorted copy + fp64 centroids):
//   adj_kernel       d(s1, s2) = (1/N) Σ eucl (fp32, R22) <= eps for all pairs as
//                    an n x n bitmap.  Warp = 32 x 32 block of pairs: lane j holds its
//                    track's N points in registers, the 32 row tracks are broadcast from
//                    shared memory; the row word is a ballot, the column word is built
//                    per lane (d is bitwise symmetric: only blocks on/above the diagonal).
//                    Exact pruning by centroid distance (block and pair level) and an
//                    exact early exit on the monotone partial sums.  ALU-bound (sqrt).
//   core_kernel      neighbour counts = row popcounts -> core flags + core bitmask.
//   cc_kernel        components of core tracks: min-original-index propagation with
//                    pointer jumping over the bitmap words, one cooperative grid.
//   roots/root_prefix/label_kernel  cluster ids by smallest original index (R23),
//                    border tracks -> smallest cluster among core neighbours, noise -1.
//   member_sort_kernel  stable counting sort of the tracks by cluster (one CTA).
//   member_gather_kernel  member rows copied into cluster order.
//   centers_kernel   warp per cluster streaming its index-ordered members through a
//                    bulk-copy (TMA) smem ring: per-point fp64 sums in that order.
//   refine_kernel    warp per 32 query tracks: each lane resamples one query into shared
//                    memory; then per query: lanes scan the
//                    cluster centres (in shared memory) with the "passes close to d1 and
//                    dn" predicate (R24) and keep a sorted top-k in registers, a warp
//                    merge picks the k nearest, 4 lanes take the weighted medians (R25).
#include <limits.h>
#include <math.h>

#include <algorithm>

#include <cooperative_groups.h>

#include "common.cuh"

namespace cg = cooperative_groups;

namespace otif {
namespace {

constexpr int kMaxPts = 32;    // N <= 32 (the paper's N = 20)
constexpr int kMaxK = 16;      // k <= 16 (the paper's k = 10)
constexpr int kMaxDbscanN = 1 << 19;

// ---- fixed-order IEEE arithmetic (readings R21, R22) -------------------------------
__device__ __forceinline__ float eucl32(float ax, float ay, float bx, float by) {
    const float dx = __fsub_rn(ax, bx), dy = __fsub_rn(ay, by);
    return __fsqrt_rn(__fadd_rn(__fmul_rn(dx, dx), __fmul_rn(dy, dy)));
}

__device__ __forceinline__ double seglen(float2 a, float2 b) {
    const double dx = __dsub_rn((double)b.x, (double)a.x), dy = __dsub_rn((double)b.y, (double)a.y);
    return __dsqrt_rn(__dadd_rn(__dmul_rn(dx, dx), __dmul_rn(dy, dy)));
}

// P:L196 / reading R21, one warp per track: cum_{j+1} = cum_j + |p_{j+1} - p_j| in order,
// point i at s = (L*i)/(N-1) on the first segment with cum_{j+1} >= s.  The lanes compute
// 32 segment lengths at a time (each independently rounded); every lane then runs the
// same sequential fp64 prefix over them (shuffles), so all lanes hold identical cum_j and
// the emitted points are the oracle's bit for bit.  Two passes (L first).  `out` may be
// global or shared memory; lane 0 writes.
__device__ void resample_track_warp(const float2 *__restrict__ p, int64_t n, int npts, float2 *out) {
    const int lane = threadIdx.x & 31;
    if (n < 1) {
        if (lane < npts)
            out[lane] = make_float2(__int_as_float(0x7fc00000), __int_as_float(0x7fc00000));
        return;
    }
    const float2 p0 = p[0];
    double L = 0.0;
    for (int64_t c0 = 0; c0 + 1 < n; c0 += 32) {
        const int64_t j = c0 + lane;
        const double seg = j + 1 < n ? seglen(p[j], p[j + 1]) : 0.0;
        const int cnt = (int)(n - 1 - c0 < 32 ? n - 1 - c0 : 32);
        for (int b = 0; b < cnt; b++) L = __dadd_rn(L, __shfl_sync(0xffffffffu, seg, b));
    }
    if (n == 1 || L == 0.0) {
        if (lane < npts) out[lane] = p0;
        return;
    }
    if (lane == 0) {
        out[0] = p0;
        out[npts - 1] = p[n - 1];
    }
    int i = 1;
    double s = __ddiv_rn(__dmul_rn(L, 1.0), (double)(npts - 1));
    double cum = 0.0;
    for (int64_t c0 = 0; c0 + 1 < n && i < npts - 1; c0 += 32) {
        const int64_t jl = c0 + lane;
        const float2 a_l = jl + 1 < n ? p[jl] : p0, b_l = jl + 1 < n ? p[jl + 1] : p0;
        const double seg = jl + 1 < n ? seglen(a_l, b_l) : 0.0;
        const int cnt = (int)(n - 1 - c0 < 32 ? n - 1 - c0 : 32);
        for (int b = 0; b < cnt && i < npts - 1; b++) {
            const double sj = __shfl_sync(0xffffffffu, seg, b);
            const double cj1 = __dadd_rn(cum, sj);
            if (!(cj1 < s)) {
                const float ax = __shfl_sync(0xffffffffu, a_l.x, b), ay = __shfl_sync(0xffffffffu, a_l.y, b);
                const float bx = __shfl_sync(0xffffffffu, b_l.x, b), by = __shfl_sync(0xffffffffu, b_l.y, b);
                do {
                    double t = __ddiv_rn(__dsub_rn(s, cum), sj);
                    if (t > 1.0) t = 1.0;
                    const double x = __dadd_rn((double)ax, __dmul_rn(t, __dsub_rn((double)bx, (double)ax)));
                    const double y = __dadd_rn((double)ay, __dmul_rn(t, __dsub_rn((double)by, (double)ay)));
                    if (lane == 0) out[i] = make_float2(__double2float_rn(x), __double2float_rn(y));
                    i++;
                    s = __ddiv_rn(__dmul_rn(L, (double)i), (double)(npts - 1));
                } while (i < npts - 1 && !(cj1 < s));
            }
            cum = cj1;
        }
    }
}

// The same procedure by one thread (the query tracks of refine_kernel are short; each lane
// resamples its own query).  Identical operations in identical order.
__device__ void resample_track_thread(const float2 *__restrict__ p, int64_t n, int npts, float2 *out) {
    if (n < 1) {
        for (int i = 0; i < npts; i++) out[i] = make_float2(__int_as_float(0x7fc00000), __int_as_float(0x7fc00000));
        return;
    }
    const float2 p0 = p[0];
    double L = 0.0;
    for (int64_t j = 0; j + 1 < n; j++) L = __dadd_rn(L, seglen(p[j], p[j + 1]));
    if (n == 1 || L == 0.0) {
        for (int i = 0; i < npts; i++) out[i] = p0;
        return;
    }
    out[0] = p0;
    int64_t j = 0;
    double cj = 0.0, sj = seglen(p[0], p[1]);
    double cj1 = __dadd_rn(cj, sj);
    for (int i = 1; i < npts - 1; i++) {
        const double sv = __ddiv_rn(__dmul_rn(L, (double)i), (double)(npts - 1));
        while (cj1 < sv) {
            j++;
            cj = cj1;
            sj = seglen(p[j], p[j + 1]);
            cj1 = __dadd_rn(cj, sj);
        }
        double t = __ddiv_rn(__dsub_rn(sv, cj), sj);
        if (t > 1.0) t = 1.0;
        const float2 a = p[j], b = p[j + 1];
        const double x = __dadd_rn((double)a.x, __dmul_rn(t, __dsub_rn((double)b.x, (double)a.x)));
        const double y = __dadd_rn((double)a.y, __dmul_rn(t, __dsub_rn((double)b.y, (double)a.y)));
        out[i] = make_float2(__double2float_rn(x), __double2float_rn(y));
    }
    out[npts - 1] = p[n - 1];
}

__global__ void resample_kernel(const float2 *__restrict__ pts, const int64_t *__restrict__ offsets, int64_t n,
                                int npts, float2 *__restrict__ P) {
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t t = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5; t < n; t += nw) {
        const int64_t o = offsets[t];
        resample_track_warp(pts + o, offsets[t + 1] - o, npts, P + t * npts);
    }
}

// ---- DBSCAN (reading R23) -----------------------------------------------------
// The work runs in a "sorted space": the tracks are ordered by (start cell, end cell,
// index) so that 32-track blocks of the neighbour bitmap are spatially coherent and whole
// blocks can be skipped.  The order only affects speed: every neighbour decision is the
// oracle's fp32 comparison, pruning is exact (below), and cluster ids are assigned by
// the smallest ORIGINAL index.
//
// Exact pruning: d(s1, s2) = (1/N) Σ |p_i - q_i| >= |mean(p) - mean(q)| (triangle
// inequality), and the fp32 d̂ >= d (1 - (N+6) 2^-24).  A pair whose fp64 centroid
// distance exceeds eps (1 + 1e-5) + 1e-6 therefore has d̂ > eps and is not evaluated.
// Early exit: partial fp32 sums of non-negative terms only grow, so once every lane's
// partial sum exceeds S* (the largest S with fl(S / N) <= eps) the row is decided.

// stable scatter of one warp's contiguous segment [lo, hi) of `src` by an 8-bit digit;
// cur = this warp's 256 running output positions
__device__ __forceinline__ void warp_stable_scatter(const int32_t *__restrict__ src, const uint16_t *__restrict__ keys,
                                                    int shift, int lo, int hi, int32_t *__restrict__ dst, int32_t *cur) {
    const int lane = threadIdx.x & 31;
    const uint32_t lt = (1u << lane) - 1u;
    for (int base = lo; base < hi; base += 32) {
        const int i = base + lane;
        const int v = i < hi ? (src ? src[i] : i) : -1;
        const int d = v >= 0 ? (keys[v] >> shift) & 255 : -1;
        const uint32_t grp = __match_any_sync(0xffffffffu, d);
        const int pos = d >= 0 ? cur[d] + __popc(grp & lt) : 0;
        __syncwarp();
        if (d >= 0) {
            dst[pos] = v;
            if ((grp & lt) == 0) cur[d] += __popc(grp);
        }
        __syncwarp();
    }
}

// one CTA: 16-bit keys (start cell << 8 | end cell on a 16 x 16 grid over the endpoints'
// bounding box), then two stable 8-bit LSD passes -> perm (sorted -> original).
__global__ void __launch_bounds__(1024) sort_kernel(const float2 *__restrict__ P, int n, int npts,
                                                    uint16_t *__restrict__ keys, int32_t *__restrict__ tmp,
                                                    int32_t *__restrict__ perm) {
    __shared__ float red[4][32];
    __shared__ int32_t hist[256];
    __shared__ int32_t whist[32][256];
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const float INF = __int_as_float(0x7f800000);
    float mnx = INF, mny = INF, mxx = -INF, mxy = -INF;
    for (int i = tid; i < n; i += blockDim.x) {
        const float2 a = P[(int64_t)i * npts], b = P[(int64_t)i * npts + npts - 1];
        mnx = fminf(mnx, fminf(a.x, b.x)); mxx = fmaxf(mxx, fmaxf(a.x, b.x));
        mny = fminf(mny, fminf(a.y, b.y)); mxy = fmaxf(mxy, fmaxf(a.y, b.y));
    }
    for (int s = 16; s > 0; s >>= 1) {
        mnx = fminf(mnx, __shfl_xor_sync(0xffffffffu, mnx, s)); mxx = fmaxf(mxx, __shfl_xor_sync(0xffffffffu, mxx, s));
        mny = fminf(mny, __shfl_xor_sync(0xffffffffu, mny, s)); mxy = fmaxf(mxy, __shfl_xor_sync(0xffffffffu, mxy, s));
    }
    if (lane == 0) { red[0][warp] = mnx; red[1][warp] = mxx; red[2][warp] = mny; red[3][warp] = mxy; }
    __syncthreads();
    mnx = red[0][0]; mxx = red[1][0]; mny = red[2][0]; mxy = red[3][0];
    for (int w = 1; w < (int)(blockDim.x >> 5); w++) {
        mnx = fminf(mnx, red[0][w]); mxx = fmaxf(mxx, red[1][w]);
        mny = fminf(mny, red[2][w]); mxy = fmaxf(mxy, red[3][w]);
    }
    const float gx = mxx > mnx ? (mxx - mnx) / 16.f : 1.f, gy = mxy > mny ? (mxy - mny) / 16.f : 1.f;
    auto cell = [&](float2 p) {
        const int cx = (int)fminf(15.f, fmaxf(0.f, (p.x - mnx) / gx));
        const int cy = (int)fminf(15.f, fmaxf(0.f, (p.y - mny) / gy));
        return cy * 16 + cx;
    };
    for (int i = tid; i < n; i += blockDim.x)
        keys[i] = (uint16_t)((cell(P[(int64_t)i * npts]) << 8) | cell(P[(int64_t)i * npts + npts - 1]));
    // two stable LSD passes; warp w owns the contiguous segment [w*seg, (w+1)*seg)
    const int nwarp = blockDim.x >> 5;
    const int seg = (n + nwarp - 1) / nwarp;
    const int lo = min(n, warp * seg), hi = min(n, lo + seg);
    __syncthreads();
    for (int pass = 0; pass < 2; pass++) {
        const int shift = pass * 8;
        const int32_t *src = pass ? tmp : nullptr;
        int32_t *dst = pass ? perm : tmp;
        for (int t = tid; t < 32 * 256; t += blockDim.x) whist[t / 256][t % 256] = 0;
        __syncthreads();
        for (int i = lo + lane; i < hi; i += 32) atomicAdd(&whist[warp][(keys[src ? src[i] : i] >> shift) & 255], 1);
        __syncthreads();
        // column prefix over warps per digit, then exclusive scan of the digit totals
        if (tid < 256) {
            int run = 0;
            for (int w = 0; w < nwarp; w++) {
                const int c = whist[w][tid];
                whist[w][tid] = run;
                run += c;
            }
            hist[tid] = run;
        }
        __syncthreads();
        if (warp == 0) {
            int v[8], loc = 0;
#pragma unroll
            for (int e = 0; e < 8; e++) { v[e] = hist[lane * 8 + e]; loc += v[e]; }
            int incl = loc;
            for (int s2 = 1; s2 < 32; s2 <<= 1) {
                const int u = __shfl_up_sync(0xffffffffu, incl, s2);
                if (lane >= s2) incl += u;
            }
            int run = incl - loc;
#pragma unroll
            for (int e = 0; e < 8; e++) { hist[lane * 8 + e] = run; run += v[e]; }
        }
        __syncthreads();
        for (int t = tid; t < 32 * 256; t += blockDim.x) whist[t / 256][t % 256] += hist[t % 256];
        __syncthreads();
        warp_stable_scatter(src, keys, shift, lo, hi, dst, whist[warp]);
        __syncthreads();
    }
}

// sorted copy of P, fp64 centroids, inverse permutation
__global__ void gather_kernel(const float2 *__restrict__ P, const int32_t *__restrict__ perm, int n, int npts,
                              float2 *__restrict__ Ps, double2 *__restrict__ cen, int32_t *__restrict__ inv) {
    for (int s = blockIdx.x * blockDim.x + threadIdx.x; s < n; s += gridDim.x * blockDim.x) {
        const int i = perm[s];
        double sx = 0.0, sy = 0.0;
        for (int q = 0; q < npts; q++) {
            const float2 p = P[(int64_t)i * npts + q];
            Ps[(int64_t)s * npts + q] = p;
            sx += (double)p.x;
            sy += (double)p.y;
        }
        cen[s] = make_double2(sx / npts, sy / npts);
        inv[i] = s;
    }
}

__device__ __forceinline__ void box_reduce(double &mnx, double &mxx, double &mny, double &mxy) {
    for (int s = 16; s > 0; s >>= 1) {
        mnx = fmin(mnx, __shfl_xor_sync(0xffffffffu, mnx, s)); mxx = fmax(mxx, __shfl_xor_sync(0xffffffffu, mxx, s));
        mny = fmin(mny, __shfl_xor_sync(0xffffffffu, mny, s)); mxy = fmax(mxy, __shfl_xor_sync(0xffffffffu, mxy, s));
    }
}

// grid (ceil(W/8), W): CTA = row block a x 8 column blocks b (one per warp), b >= a.
template <int NP>
__global__ void __launch_bounds__(256) adj_kernel(const float2 *__restrict__ Ps, const double2 *__restrict__ cen, int n,
                                                  int npts, float smax, double thr, uint32_t *__restrict__ adj,
                                                  int pitch) {
    const int a = blockIdx.y;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if ((int)blockIdx.x * 8 + 7 < a) return;          // whole CTA below the diagonal
    __shared__ float2 si[32][NP];
    __shared__ double2 ci[32];
    __shared__ double ibox[4];
    for (int t = threadIdx.x; t < 32 * npts; t += blockDim.x) {
        const int r = t / npts, q = t - r * npts, i = a * 32 + r;
        si[r][q] = i < n ? Ps[(int64_t)i * npts + q] : make_float2(0.f, 0.f);
    }
    const double DINF = __longlong_as_double(0x7ff0000000000000LL);
    if (warp == 0) {
        const int i = a * 32 + lane;
        const double2 c = i < n ? cen[i] : make_double2(0.0, 0.0);
        ci[lane] = c;
        double mnx = i < n ? c.x : DINF, mxx = i < n ? c.x : -DINF, mny = i < n ? c.y : DINF, mxy = i < n ? c.y : -DINF;
        box_reduce(mnx, mxx, mny, mxy);
        if (lane == 0) { ibox[0] = mnx; ibox[1] = mxx; ibox[2] = mny; ibox[3] = mxy; }
    }
    __syncthreads();
    const int b = blockIdx.x * 8 + warp;
    if (b < a || b * 32 >= n) return;
    const int j = b * 32 + lane;
    const double2 cj = j < n ? cen[j] : make_double2(0.0, 0.0);
    {
        double mnx = j < n ? cj.x : DINF, mxx = j < n ? cj.x : -DINF, mny = j < n ? cj.y : DINF,
               mxy = j < n ? cj.y : -DINF;
        box_reduce(mnx, mxx, mny, mxy);
        const double gx = fmax(0.0, fmax(ibox[0] - mxx, mnx - ibox[1]));
        const double gy = fmax(0.0, fmax(ibox[2] - mxy, mny - ibox[3]));
        if (gx * gx + gy * gy > thr * thr) return;    // no pair of the block can be neighbours
    }
    float2 pj[NP];
#pragma unroll
    for (int q = 0; q < NP; q++) pj[q] = (j < n && q < npts) ? Ps[(int64_t)j * npts + q] : make_float2(0.f, 0.f);
    const float INF = __int_as_float(0x7f800000);
    const double thr2 = thr * thr;
    const int rows = min(32, n - a * 32);
    uint32_t col = 0;
    for (int r = 0; r < rows; r++) {
        const double dx = ci[r].x - cj.x, dy = ci[r].y - cj.y;
        const bool live = j < n && dx * dx + dy * dy <= thr2;
        if (!__any_sync(0xffffffffu, live)) continue;
        float sum = live ? 0.f : INF;
        bool done = false;                             // warp-uniform
#pragma unroll
        for (int q = 0; q < NP; q++) {
            if (!done && (NP != kMaxPts || q < npts)) {
                const float2 x = si[r][q];
                sum = __fadd_rn(sum, eucl32(x.x, x.y, pj[q].x, pj[q].y));
                if ((q & 3) == 3) done = __all_sync(0xffffffffu, sum > smax);
            }
        }
        const bool nb = sum <= smax;
        const uint32_t row = __ballot_sync(0xffffffffu, nb);
        if (lane == 0 && row) adj[(int64_t)(a * 32 + r) * pitch + b] = row;
        col |= (uint32_t)nb << r;
    }
    if (a != b && j < n && col) adj[(int64_t)j * pitch + a] = col;
}

// core flag = |neighbours| >= min_pts (sorted space); outputs core in original order,
// the sorted core bitmask and the initial component keys (original index).
__global__ void __launch_bounds__(1024) core_kernel(const uint32_t *__restrict__ adj, const int32_t *__restrict__ perm,
                                                    int n, int W, int pitch, int min_pts, uint8_t *__restrict__ core,
                                                    uint32_t *__restrict__ coremask, int32_t *__restrict__ lab) {
    __shared__ uint32_t flag[32];
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int s = blockIdx.x * 32 + warp;
    int cnt = 0;
    if (s < n)
        for (int w = lane; w < W; w += 32) cnt += __popc(adj[(int64_t)s * pitch + w]);
    for (int k = 16; k > 0; k >>= 1) cnt += __shfl_xor_sync(0xffffffffu, cnt, k);
    const bool c = s < n && cnt >= min_pts;
    if (lane == 0) {
        flag[warp] = c;
        lab[s] = c ? perm[s] : INT_MAX;            // lab is padded to 32 * W entries
        if (s < n && core) core[perm[s]] = c;
    }
    __syncthreads();
    if (warp == 0) {
        const uint32_t m = __ballot_sync(0xffffffffu, flag[lane] != 0);
        if (lane == 0) coremask[blockIdx.x] = m;
    }
}

// min over the core neighbours' keys of one sorted row (word-level: 8 x 16-B loads of the
// 32 keys of a word with any core neighbour)
__device__ __forceinline__ int row_min_key(const uint32_t *__restrict__ row, const uint32_t *__restrict__ coremask,
                                           const int32_t *lab, int W, int best) {
    const int lane = threadIdx.x & 31;
    for (int w = lane; w < W; w += 32) {
        const uint32_t m = row[w] & coremask[w];
        if (!m) continue;
        const int4 *L4 = reinterpret_cast<const int4 *>(lab + 32 * w);
#pragma unroll
        for (int v = 0; v < 8; v++) {
            if (!((m >> (4 * v)) & 15u)) continue;
            const int4 x = __ldcg(L4 + v);
            if ((m >> (4 * v)) & 1u) best = min(best, x.x);
            if ((m >> (4 * v + 1)) & 1u) best = min(best, x.y);
            if ((m >> (4 * v + 2)) & 1u) best = min(best, x.z);
            if ((m >> (4 * v + 3)) & 1u) best = min(best, x.w);
        }
    }
    for (int k = 16; k > 0; k >>= 1) best = min(best, __shfl_xor_sync(0xffffffffu, best, k));
    return best;
}

// Connected components of the core tracks by min-key propagation with pointer jumping
// (a core track's key -> the smallest original index in its component), one persistent
// cooperative grid; iterates until a pass changes nothing.  A pass only reads the keys of
// neighbour words that changed in the previous pass (chg bitmasks, rotating by 3 like the
// flags); each lane loads 4 bitmap words at a time.
__global__ void __launch_bounds__(256) cc_kernel(const uint32_t *__restrict__ adj, const uint32_t *__restrict__ coremask,
                                                 const int32_t *__restrict__ inv, int n, int W, int pitch,
                                                 int32_t *lab, int32_t *flags, uint32_t *chg) {
    cg::grid_group grid = cg::this_grid();
    extern __shared__ uint32_t ccm[];                 // coremask copy [pitch]
    for (int w = threadIdx.x; w < pitch; w += blockDim.x) ccm[w] = w < W ? coremask[w] : 0u;
    __syncthreads();
    const int lane = threadIdx.x & 31;
    const int64_t gw = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int it = 0;; it++) {
        int32_t *flag = flags + (it % 3);
        const uint32_t *prev = chg + (size_t)((it + 2) % 3) * pitch;   // changed in pass it-1
        uint32_t *cur = chg + (size_t)(it % 3) * pitch;
        uint32_t *nxt = chg + (size_t)((it + 1) % 3) * pitch;
        if (grid.thread_rank() == 0) flags[(it + 1) % 3] = 0;
        for (int64_t w = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; w < pitch; w += (int64_t)gridDim.x * blockDim.x)
            nxt[w] = 0u;
        for (int64_t s = gw; s < n; s += nw) {
            if (!((ccm[s >> 5] >> (s & 31)) & 1u)) continue;
            const int own = __ldcg(lab + s);
            const int j1 = __ldcg(lab + inv[own]);
            const int j2 = __ldcg(lab + inv[j1]);
            int best = min(own, min(j1, j2));
            const uint32_t *row = adj + s * pitch;
#pragma unroll 2
            for (int base = lane * 4; base < pitch; base += 128) {
                const uint4 r = __ldcg(reinterpret_cast<const uint4 *>(row + base));
                const uint4 ch = it ? __ldcg(reinterpret_cast<const uint4 *>(prev + base)) : make_uint4(~0u, ~0u, ~0u, ~0u);
                const uint32_t mm[4] = {r.x & ccm[base] & ch.x, r.y & ccm[base + 1] & ch.y, r.z & ccm[base + 2] & ch.z,
                                        r.w & ccm[base + 3] & ch.w};
#pragma unroll
                for (int e = 0; e < 4; e++) {
                    const uint32_t m = mm[e];
                    if (!m) continue;
                    const int4 *L4 = reinterpret_cast<const int4 *>(lab + 32 * (base + e));
#pragma unroll
                    for (int v = 0; v < 8; v++) {
                        if (!((m >> (4 * v)) & 15u)) continue;
                        const int4 x = __ldcg(L4 + v);
                        if ((m >> (4 * v)) & 1u) best = min(best, x.x);
                        if ((m >> (4 * v + 1)) & 1u) best = min(best, x.y);
                        if ((m >> (4 * v + 2)) & 1u) best = min(best, x.z);
                        if ((m >> (4 * v + 3)) & 1u) best = min(best, x.w);
                    }
                }
            }
            for (int k = 16; k > 0; k >>= 1) best = min(best, __shfl_xor_sync(0xffffffffu, best, k));
            if (lane == 0 && best < own) {
                atomicMin(lab + s, best);
                atomicOr(cur + (s >> 5), 1u << (s & 31));
                *flag = 1;
            }
        }
        grid.sync();
        if (*(volatile int32_t *)flag == 0) {
            if (grid.thread_rank() == 0) flags[3] = it + 1;     // passes, for diagnostics
            break;
        }
    }
}

// cluster roots (tracks whose key is their own original index) as bits in original space
__global__ void roots_kernel(const int32_t *__restrict__ lab, const int32_t *__restrict__ perm,
                             const uint32_t *__restrict__ coremask, int n, uint32_t *__restrict__ rootbits) {
    for (int s = blockIdx.x * blockDim.x + threadIdx.x; s < n; s += gridDim.x * blockDim.x) {
        if (!((coremask[s >> 5] >> (s & 31)) & 1u)) continue;
        const int i = perm[s];
        if (lab[s] == i) atomicOr(rootbits + (i >> 5), 1u << (i & 31));
    }
}

// exclusive prefix of the root counts per word (one CTA) -> cluster id of a root key
__global__ void __launch_bounds__(1024) root_prefix_kernel(const uint32_t *__restrict__ rootbits, int W,
                                                           int32_t *__restrict__ wprefix,
                                                           int32_t *__restrict__ n_clusters) {
    __shared__ int32_t part[32];
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const int per = (W + blockDim.x - 1) / blockDim.x;
    const int lo = min(W, tid * per), hi = min(W, lo + per);
    int local = 0;
    for (int w = lo; w < hi; w++) local += __popc(rootbits[w]);
    int incl = local;
    for (int s = 1; s < 32; s <<= 1) {
        const int u = __shfl_up_sync(0xffffffffu, incl, s);
        if (lane >= s) incl += u;
    }
    if (lane == 31) part[warp] = incl;
    __syncthreads();
    if (warp == 0) {
        int v = part[lane];
        for (int s = 1; s < 32; s <<= 1) {
            const int u = __shfl_up_sync(0xffffffffu, v, s);
            if (lane >= s) v += u;
        }
        part[lane] = v;
    }
    __syncthreads();
    int run = (warp ? part[warp - 1] : 0) + incl - local;
    for (int w = lo; w < hi; w++) {
        wprefix[w] = run;
        run += __popc(rootbits[w]);
    }
    if (tid == 0) *n_clusters = part[31];
}

__device__ __forceinline__ int cluster_of(int key, const uint32_t *__restrict__ rootbits,
                                          const int32_t *__restrict__ wprefix) {
    return wprefix[key >> 5] + __popc(rootbits[key >> 5] & ((1u << (key & 31)) - 1u));
}

// labels in original order: core -> cluster of its key; border -> smallest cluster among
// its core neighbours (= cluster of the smallest neighbour key); noise -1.
__global__ void label_kernel(const uint32_t *__restrict__ adj, const uint32_t *__restrict__ coremask,
                             const int32_t *__restrict__ perm, const int32_t *lab,
                             const uint32_t *__restrict__ rootbits, const int32_t *__restrict__ wprefix, int n, int W,
                             int pitch, int32_t *__restrict__ labels) {
    const int lane = threadIdx.x & 31;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t s = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5; s < n; s += nw) {
        if ((coremask[s >> 5] >> (s & 31)) & 1u) {
            if (lane == 0) labels[perm[s]] = cluster_of(lab[s], rootbits, wprefix);
            continue;
        }
        const int best = row_min_key(adj + s * pitch, coremask, lab, W, INT_MAX);
        if (lane == 0) labels[perm[s]] = best == INT_MAX ? -1 : cluster_of(best, rootbits, wprefix);
    }
}

// Stable member order (counting sort by label, index order inside a label), one CTA:
// per-label counts -> exclusive scan -> one warp scatters in index order, ranks from
// __match_any_sync.  Cursors live in shared memory when nc fits, else in the workspace.
__global__ void __launch_bounds__(1024) member_sort_kernel(const int32_t *__restrict__ labels, int64_t n, int nc,
                                                           int32_t *__restrict__ order, int32_t *__restrict__ start,
                                                           int32_t *__restrict__ sizes, int32_t *__restrict__ gcur,
                                                           int use_smem) {
    extern __shared__ int32_t msm[];
    __shared__ int32_t part[33];
    int32_t *cur = use_smem ? msm : gcur;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    for (int c = tid; c < nc; c += blockDim.x) cur[c] = 0;
    __syncthreads();
    for (int64_t i = tid; i < n; i += blockDim.x) {
        const int lab = labels[i];
        if (lab >= 0 && lab < nc) atomicAdd(&cur[lab], 1);
    }
    __syncthreads();
    // exclusive scan over nc: thread t owns the contiguous range [t*per, (t+1)*per)
    const int per = (nc + blockDim.x - 1) / blockDim.x;
    const int lo = min(nc, tid * per), hi = min(nc, lo + per);
    int local = 0;
    for (int c = lo; c < hi; c++) local += cur[c];
    int incl = local;
    for (int s = 1; s < 32; s <<= 1) {
        const int v = __shfl_up_sync(0xffffffffu, incl, s);
        if (lane >= s) incl += v;
    }
    if (lane == 31) part[warp] = incl;
    __syncthreads();
    if (warp == 0) {
        int v = lane < (int)(blockDim.x >> 5) ? part[lane] : 0;
        for (int s = 1; s < 32; s <<= 1) {
            const int u = __shfl_up_sync(0xffffffffu, v, s);
            if (lane >= s) v += u;
        }
        part[lane] = v;            // inclusive warp totals
    }
    __syncthreads();
    int run = (warp ? part[warp - 1] : 0) + incl - local;
    for (int c = lo; c < hi; c++) {
        const int k = cur[c];
        start[c] = run;
        sizes[c] = k;
        cur[c] = run;
        run += k;
    }
    if (tid == 0) start[nc] = part[31];
    __syncthreads();
    if (warp != 0) return;
    const uint32_t lt = (1u << lane) - 1u;
    for (int64_t base = 0; base < n; base += 32) {
        const int64_t i = base + lane;
        int lab = i < n ? labels[i] : -1;
        if (lab >= nc) lab = -1;
        const uint32_t grp = __match_any_sync(0xffffffffu, lab);
        const int pos = lab >= 0 ? cur[lab] + __popc(grp & lt) : 0;
        __syncwarp();
        if (lab >= 0) {
            order[pos] = (int32_t)i;
            if ((grp & lt) == 0) cur[lab] += __popc(grp);
        }
        __syncwarp();
    }
}

// member rows in cluster order: Pm[pos] = P[order[pos]] (fully parallel)
__global__ void member_gather_kernel(const float *__restrict__ P, const int32_t *__restrict__ order,
                                     const int32_t *__restrict__ start, int nc, int q2, float *__restrict__ Pm) {
    const int64_t total = (int64_t)start[nc] * q2;
    for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < total; e += (int64_t)gridDim.x * blockDim.x) {
        const int64_t pos = e / q2;
        Pm[e] = P[(int64_t)order[pos] * q2 + (e - pos * q2)];
    }
}

constexpr int kCenterRows = 32;     // rows per bulk-copy chunk
constexpr int kCenterStages = 4;

// P:L198 centres: one warp (CTA) per cluster streams its index-ordered member rows
// (contiguous in Pm) through a 4-stage shared-memory ring filled by 1-D bulk copies
// (TMA engine, mbarrier completion); lanes add their coordinates in fp64 in row order.
__global__ void __launch_bounds__(32) centers_kernel(const float *__restrict__ Pm, const int32_t *__restrict__ start,
                                                     int npts, int nc, float *__restrict__ centers) {
    extern __shared__ __align__(128) float csm[];                 // [stages][rows][q2]
    __shared__ __align__(8) uint64_t bars[kCenterStages];
    const int lane = threadIdx.x;
    const int c = blockIdx.x;
    const int q2 = 2 * npts;
    const int s = start[c], cnt = start[c + 1] - s;
    const float *rows = Pm + (int64_t)s * q2;
    const int nchunk = (cnt + kCenterRows - 1) / kCenterRows;
    if (lane == 0) {
        for (int k = 0; k < kCenterStages; k++) mbar_init(&bars[k], 1);
        fence_barrier_init();
    }
    __syncwarp();
    auto issue = [&](int ch) {
        const int st = ch % kCenterStages;
        const int nr = min(kCenterRows, cnt - ch * kCenterRows);
        const uint32_t bytes = (uint32_t)nr * q2 * 4;
        mbar_arrive_expect_tx(&bars[st], bytes);
        bulk_g2s(csm + (size_t)st * kCenterRows * q2, rows + (int64_t)ch * kCenterRows * q2, bytes, &bars[st]);
    };
    if (lane == 0)
        for (int ch = 0; ch < min(nchunk, kCenterStages); ch++) issue(ch);
    double s0 = 0.0, s1 = 0.0;
    for (int ch = 0; ch < nchunk; ch++) {
        const int st = ch % kCenterStages;
        mbar_wait(&bars[st], (uint32_t)((ch / kCenterStages) & 1));
        const float *buf = csm + (size_t)st * kCenterRows * q2;
        const int nr = min(kCenterRows, cnt - ch * kCenterRows);
        for (int r = 0; r < nr; r++) {
            if (lane < q2) s0 = __dadd_rn(s0, (double)buf[r * q2 + lane]);
            if (lane + 32 < q2) s1 = __dadd_rn(s1, (double)buf[r * q2 + lane + 32]);
        }
        __syncwarp();
        if (lane == 0 && ch + kCenterStages < nchunk) issue(ch + kCenterStages);
    }
    const double dc = (double)cnt;
    if (lane < q2) centers[(int64_t)c * q2 + lane] = cnt ? __double2float_rn(__ddiv_rn(s0, dc)) : 0.f;
    if (lane + 32 < q2) centers[(int64_t)c * q2 + lane + 32] = cnt ? __double2float_rn(__ddiv_rn(s1, dc)) : 0.f;
}

// ---- refinement ---------------------------------------------------------------------
__device__ __forceinline__ bool lex_less(float d, int c, float d2, int c2) {
    return d < d2 || (d == d2 && c < c2);
}

// shared-memory centre pitch in floats: 2*(npts+1) or 2*(npts+2), whichever has an odd
// number of float2 -> 16 lanes' 8-byte loads of 16 different centres hit distinct banks
__host__ __device__ inline int center_pitch(int npts) { return ((npts + 1) & 1) ? 2 * (npts + 1) : 2 * (npts + 2); }

constexpr int kRefineWarps = 8;

__global__ void __launch_bounds__(kRefineWarps * 32) refine_kernel(
    const float2 *__restrict__ pts, const int64_t *__restrict__ offsets, int64_t m, int npts,
    const float *__restrict__ centers, const int32_t *__restrict__ sizes, int nc, int k, float rho,
    float *__restrict__ out, int32_t *__restrict__ used) {
    extern __shared__ float rsm[];
    const int pitch = center_pitch(npts);
    float *sC = rsm;                                                    // [nc][pitch]
    int32_t *sW = reinterpret_cast<int32_t *>(sC + (size_t)nc * pitch); // [nc]
    float2 *sQ = reinterpret_cast<float2 *>(sW + ((nc + 1) & ~1));      // [warps][32][npts]
    for (int t = threadIdx.x; t < nc * 2 * npts; t += blockDim.x) {
        const int c = t / (2 * npts), q = t - c * 2 * npts;
        sC[c * pitch + q] = centers[t];
    }
    for (int t = threadIdx.x; t < nc; t += blockDim.x) sW[t] = sizes[t];
    __syncthreads();
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    float2 *wQ = sQ + (size_t)warp * 32 * npts;
    const float fn = (float)npts;
    const float INF = __int_as_float(0x7f800000);
    for (int64_t q0 = ((int64_t)blockIdx.x * kRefineWarps + warp) * 32; q0 < m;
         q0 += (int64_t)gridDim.x * kRefineWarps * 32) {
        // each lane resamples one query of the batch of 32
        float2 l1 = make_float2(0.f, 0.f), ln = make_float2(0.f, 0.f);
        int64_t llen = 0;
        if (q0 + lane < m) {
            const int64_t o = offsets[q0 + lane];
            llen = offsets[q0 + lane + 1] - o;
            resample_track_thread(pts + o, llen, npts, wQ + lane * npts);
            if (llen > 0) {
                l1 = pts[o];
                ln = pts[o + llen - 1];
            }
        }
        __syncwarp();
        const int nq = (int)(m - q0 < 32 ? m - q0 : 32);
        for (int qi = 0; qi < nq; qi++) {
            const int64_t q = q0 + qi;
            const float2 *myQ = wQ + qi * npts;
            const float2 d1 = make_float2(__shfl_sync(0xffffffffu, l1.x, qi), __shfl_sync(0xffffffffu, l1.y, qi));
            const float2 dn = make_float2(__shfl_sync(0xffffffffu, ln.x, qi), __shfl_sync(0xffffffffu, ln.y, qi));
            float kd[kMaxK];
            int kc[kMaxK];
#pragma unroll
            for (int t = 0; t < kMaxK; t++) { kd[t] = INF; kc[t] = INT_MAX; }
            for (int c = lane; c < nc; c += 32) {
                const float2 *cen = reinterpret_cast<const float2 *>(sC + c * pitch);
                if (rho > 0.f) {
                    bool n1 = false, n2 = false;
                    for (int i = 0; i < npts && !n1; i++) n1 = eucl32(cen[i].x, cen[i].y, d1.x, d1.y) <= rho;
                    if (!n1) continue;
                    for (int i = 0; i < npts && !n2; i++) n2 = eucl32(cen[i].x, cen[i].y, dn.x, dn.y) <= rho;
                    if (!n2) continue;
                }
                float sum = 0.f;
                for (int i = 0; i < npts; i++) sum = __fadd_rn(sum, eucl32(myQ[i].x, myQ[i].y, cen[i].x, cen[i].y));
                const float d = __fdiv_rn(sum, fn);
                if (!lex_less(d, c, kd[kMaxK - 1], kc[kMaxK - 1])) continue;
                bool placed = false;
#pragma unroll
                for (int t = kMaxK - 1; t > 0; t--) {
                    if (!placed) {
                        if (lex_less(d, c, kd[t - 1], kc[t - 1])) {
                            kd[t] = kd[t - 1];
                            kc[t] = kc[t - 1];
                        } else {
                            kd[t] = d;
                            kc[t] = c;
                            placed = true;
                        }
                    }
                }
                if (!placed) { kd[0] = d; kc[0] = c; }
            }
            // warp merge of the sorted per-lane lists: k rounds of a lexicographic argmin
            int mysel = -1, nk = 0;
            for (int r = 0; r < k; r++) {
                float bd = kd[0];
                int bc = kc[0];
                for (int s = 16; s > 0; s >>= 1) {
                    const float od = __shfl_xor_sync(0xffffffffu, bd, s);
                    const int oc = __shfl_xor_sync(0xffffffffu, bc, s);
                    if (lex_less(od, oc, bd, bc)) { bd = od; bc = oc; }
                }
                if (bc == INT_MAX) break;
                if (lane == r) mysel = bc;
                nk++;
                if (kc[0] == bc) {
#pragma unroll
                    for (int t = 0; t < kMaxK - 1; t++) { kd[t] = kd[t + 1]; kc[t] = kc[t + 1]; }
                    kd[kMaxK - 1] = INF;
                    kc[kMaxK - 1] = INT_MAX;
                }
            }
            // weighted medians: lane e < 4 takes coordinate e (start x, start y, end x, end y)
            const int e = lane & 3;
            const int off = e < 2 ? e : 2 * (npts - 1) + (e - 2);
            float v[kMaxK];
            int64_t w[kMaxK];
            int64_t total = 0;
#pragma unroll
            for (int a = 0; a < kMaxK; a++) {
                const int ca = __shfl_sync(0xffffffffu, mysel, a);
                v[a] = a < nk ? sC[ca * pitch + off] : INF;
                w[a] = a < nk ? (int64_t)sW[ca] : 0;
                total += w[a];
            }
            float best = INF;
#pragma unroll
            for (int a = 0; a < kMaxK; a++) {
                int64_t wle = 0;
#pragma unroll
                for (int b = 0; b < kMaxK; b++) wle += (v[b] <= v[a]) ? w[b] : 0;
                if (a < nk && 2 * wle >= total && v[a] < best) best = v[a];
            }
            if (lane < 4) {
                const float own = e == 0 ? d1.x : e == 1 ? d1.y : e == 2 ? dn.x : dn.y;
                out[q * 4 + e] = nk ? best : own;
            }
            if (lane == 0) used[q] = nk;
        }
        __syncwarp();
    }
}

inline bool aligned8(const void *p) { return (reinterpret_cast<uintptr_t>(p) & 7) == 0; }

inline int dbscan_pitch(int64_t n) { return (int)round_up(cdiv(n, 32), 4); }

}  // namespace
}  // namespace otif

using namespace otif;

extern "C" otif_status otif_track_resample(const float *pts, const int64_t *offsets, int64_t n, int32_t npts, float *P,
                                           cudaStream_t stream) {
    OTIF_REQUIRE(n >= 0 && npts >= 2 && npts <= kMaxPts, "otif_track_resample: n=%lld npts=%d (2..%d)",
                 (long long)n, npts, kMaxPts);
    if (n == 0) return OTIF_OK;
    OTIF_REQUIRE(pts && offsets && P, "otif_track_resample: NULL argument");
    OTIF_REQUIRE(aligned8(pts) && aligned8(P), "otif_track_resample: pts and P must be 8-byte aligned");
    int sms = 0;
    otif_status st = check_device(&sms);
    if (st != OTIF_OK) return st;
    const int threads = 256;
    const int64_t blocks = std::min<int64_t>(cdiv(n, threads / 32), (int64_t)sms * 8);
    resample_kernel<<<(unsigned)blocks, threads, 0, stream>>>(reinterpret_cast<const float2 *>(pts), offsets, n, npts,
                                                             reinterpret_cast<float2 *>(P));
    OTIF_LAUNCH_CHECK();
    return OTIF_OK;
}

namespace otif {
namespace {
// workspace layout of otif_track_dbscan (all offsets 256-B aligned)
struct DbscanLayout {
    size_t adj, coremask, perm, tmp, inv, Ps, cen, lab, keys, rootbits, wprefix, flags, chg, total;
    DbscanLayout(int64_t n, int npts) {
        const int64_t pitch = dbscan_pitch(n), W = cdiv(n, 32);
        size_t o = 0;
        auto take = [&](int64_t bytes) { size_t at = o; o += (size_t)round_up(bytes > 0 ? bytes : 1, 256); return at; };
        adj = take(n * pitch * 4);
        coremask = take(pitch * 4);
        perm = take(n * 4);
        tmp = take(n * 4);
        inv = take(n * 4);
        Ps = take(n * npts * 8);
        cen = take(n * 16);
        lab = take(32 * pitch * 4);
        keys = take(n * 2);
        rootbits = take(pitch * 4);
        wprefix = take((W + 1) * 4);
        flags = take(16);
        chg = take(3 * pitch * 4);
        total = o;
    }
};

// S* = the largest float S with fl(S / N) <= eps (IEEE single division, as on the device):
// fl(sum / N) <= eps  <=>  sum <= S* for every float sum, because division is monotone.
float sum_threshold(float eps, int npts) {
    const float fn = (float)npts;
    if (!(eps == eps)) return eps;                      // NaN: nothing is a neighbour
    if (eps == INFINITY) return INFINITY;
    volatile float s = eps * fn;
    while (s / fn > eps) s = nextafterf(s, -INFINITY);
    while (nextafterf(s, INFINITY) / fn <= eps) s = nextafterf(s, INFINITY);
    return s;
}
}  // namespace
}  // namespace otif

extern "C" size_t otif_dbscan_workspace_bytes(int64_t n) {
    if (n < 0 || n > kMaxDbscanN) return 0;
    return DbscanLayout(n, kMaxPts).total;
}

extern "C" otif_status otif_track_dbscan(const float *P, int64_t n, int32_t npts, float eps, int32_t min_pts,
                                         int32_t *labels, uint8_t *core, int32_t *n_clusters, void *workspace,
                                         size_t ws_bytes, cudaStream_t stream) {
    OTIF_REQUIRE(n >= 0 && n <= kMaxDbscanN, "otif_track_dbscan: n=%lld (0..%d)", (long long)n, kMaxDbscanN);
    OTIF_REQUIRE(npts >= 2 && npts <= kMaxPts && min_pts >= 1, "otif_track_dbscan: npts=%d min_pts=%d", npts,
                 min_pts);
    OTIF_REQUIRE(n_clusters, "otif_track_dbscan: NULL n_clusters");
    OTIF_REQUIRE(n == 0 || (P && labels && workspace), "otif_track_dbscan: NULL argument");
    OTIF_REQUIRE(n == 0 || aligned8(P), "otif_track_dbscan: P must be 8-byte aligned");
    OTIF_REQUIRE(n == 0 || (reinterpret_cast<uintptr_t>(workspace) & 255) == 0,
                 "otif_track_dbscan: workspace must be 256-byte aligned");
    OTIF_REQUIRE(ws_bytes >= otif_dbscan_workspace_bytes(n) || n == 0, "otif_track_dbscan: workspace %zu < %zu",
                 ws_bytes, otif_dbscan_workspace_bytes(n));
    int sms = 0;
    otif_status st = check_device(&sms);
    if (st != OTIF_OK) return st;
    if (n == 0) {
        OTIF_CUDA(cudaMemsetAsync(n_clusters, 0, 4, stream));
        return OTIF_OK;
    }
    const int ni = (int)n, W = (int)cdiv(n, 32), pitch = dbscan_pitch(n);
    const DbscanLayout L(n, npts);
    char *w = static_cast<char *>(workspace);
    uint32_t *adj = reinterpret_cast<uint32_t *>(w + L.adj);
    uint32_t *coremask = reinterpret_cast<uint32_t *>(w + L.coremask);
    int32_t *perm = reinterpret_cast<int32_t *>(w + L.perm);
    int32_t *tmp = reinterpret_cast<int32_t *>(w + L.tmp);
    int32_t *inv = reinterpret_cast<int32_t *>(w + L.inv);
    float2 *Ps = reinterpret_cast<float2 *>(w + L.Ps);
    double2 *cen = reinterpret_cast<double2 *>(w + L.cen);
    int32_t *lab = reinterpret_cast<int32_t *>(w + L.lab);
    uint16_t *keys = reinterpret_cast<uint16_t *>(w + L.keys);
    uint32_t *rootbits = reinterpret_cast<uint32_t *>(w + L.rootbits);
    int32_t *wprefix = reinterpret_cast<int32_t *>(w + L.wprefix);
    int32_t *flags = reinterpret_cast<int32_t *>(w + L.flags);
    uint32_t *chg = reinterpret_cast<uint32_t *>(w + L.chg);
    OTIF_CUDA(cudaMemsetAsync(adj, 0, (size_t)n * pitch * 4, stream));
    OTIF_CUDA(cudaMemsetAsync(coremask, 0, (size_t)pitch * 4, stream));
    OTIF_CUDA(cudaMemsetAsync(lab, 0x7f, (size_t)32 * pitch * 4, stream));   // padding keys: large
    OTIF_CUDA(cudaMemsetAsync(rootbits, 0, (size_t)pitch * 4, stream));
    OTIF_CUDA(cudaMemsetAsync(flags, 0, 16, stream));
    OTIF_CUDA(cudaMemsetAsync(chg, 0, (size_t)3 * pitch * 4, stream));
    const float2 *P2 = reinterpret_cast<const float2 *>(P);
    sort_kernel<<<1, 1024, 0, stream>>>(P2, ni, npts, keys, tmp, perm);
    OTIF_LAUNCH_CHECK();
    gather_kernel<<<(unsigned)std::min<int64_t>(cdiv(n, 256), (int64_t)sms * 8), 256, 0, stream>>>(P2, perm, ni, npts,
                                                                                                  Ps, cen, inv);
    OTIF_LAUNCH_CHECK();
    const float smax = sum_threshold(eps, npts);
    const double thr = (double)eps * 1.00001 + 1e-6;
    const dim3 grid((unsigned)cdiv(W, 8), (unsigned)W);
    if (npts == 20)
        adj_kernel<20><<<grid, 256, 0, stream>>>(Ps, cen, ni, npts, smax, thr, adj, pitch);
    else
        adj_kernel<kMaxPts><<<grid, 256, 0, stream>>>(Ps, cen, ni, npts, smax, thr, adj, pitch);
    OTIF_LAUNCH_CHECK();
    core_kernel<<<W, 1024, 0, stream>>>(adj, perm, ni, W, pitch, min_pts, core, coremask, lab);
    OTIF_LAUNCH_CHECK();
    const size_t cc_smem = (size_t)pitch * 4;
    if (cc_smem > 48 * 1024)
        OTIF_CUDA(cudaFuncSetAttribute(cc_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)cc_smem));
    int per_sm = 0;
    OTIF_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, cc_kernel, 256, cc_smem));
    const int cc_blocks = (int)std::min<int64_t>((int64_t)sms * std::max(per_sm, 1), cdiv(n, 8));
    int a_n = ni, a_W = W, a_pitch = pitch;
    void *args[] = {(void *)&adj, (void *)&coremask, (void *)&inv, (void *)&a_n, (void *)&a_W, (void *)&a_pitch,
                    (void *)&lab, (void *)&flags, (void *)&chg};
    OTIF_CUDA(cudaLaunchCooperativeKernel((const void *)cc_kernel, dim3(cc_blocks), dim3(256), args, cc_smem, stream));
    roots_kernel<<<(unsigned)std::min<int64_t>(cdiv(n, 256), (int64_t)sms * 8), 256, 0, stream>>>(lab, perm, coremask,
                                                                                                 ni, rootbits);
    OTIF_LAUNCH_CHECK();
    root_prefix_kernel<<<1, 1024, 0, stream>>>(rootbits, W, wprefix, n_clusters);
    OTIF_LAUNCH_CHECK();
    label_kernel<<<sms * 8, 256, 0, stream>>>(adj, coremask, perm, lab, rootbits, wprefix, ni, W, pitch, labels);
    OTIF_LAUNCH_CHECK();
    return OTIF_OK;
}

extern "C" size_t otif_centers_workspace_bytes(int64_t n, int32_t nc) {
    if (n < 0 || nc < 0 || n > INT_MAX) return 0;
    return (size_t)round_up(n * 4, 256) + (size_t)round_up((int64_t)(nc + 1) * 4, 256) +
           (size_t)round_up((int64_t)nc * 4, 256) + (size_t)round_up(n * kMaxPts * 8, 256);
}

extern "C" otif_status otif_track_centers(const float *P, const int32_t *labels, int64_t n, int32_t npts, int32_t nc,
                                          float *centers, int32_t *sizes, void *workspace, size_t ws_bytes,
                                          cudaStream_t stream) {
    OTIF_REQUIRE(n >= 0 && n <= INT_MAX && nc >= 0 && npts >= 2 && npts <= kMaxPts,
                 "otif_track_centers: n=%lld nc=%d npts=%d", (long long)n, nc, npts);
    if (nc == 0) return OTIF_OK;
    OTIF_REQUIRE(centers && sizes && workspace && (n == 0 || (P && labels)), "otif_track_centers: NULL argument");
    OTIF_REQUIRE(ws_bytes >= otif_centers_workspace_bytes(n, nc), "otif_track_centers: workspace %zu < %zu", ws_bytes,
                 otif_centers_workspace_bytes(n, nc));
    int sms = 0;
    otif_status st = check_device(&sms);
    if (st != OTIF_OK) return st;
    char *w = static_cast<char *>(workspace);
    int32_t *order = reinterpret_cast<int32_t *>(w);
    size_t o = round_up(n * 4, 256);
    int32_t *start = reinterpret_cast<int32_t *>(w + o);
    o += round_up((int64_t)(nc + 1) * 4, 256);
    int32_t *gcur = reinterpret_cast<int32_t *>(w + o);
    o += round_up((int64_t)nc * 4, 256);
    float *Pm = reinterpret_cast<float *>(w + o);
    const size_t cur_bytes = (size_t)nc * 4;
    const int use_smem = cur_bytes <= 160 * 1024;
    const size_t smem = use_smem ? cur_bytes : 0;
    if (smem > 48 * 1024)
        OTIF_CUDA(cudaFuncSetAttribute(member_sort_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    member_sort_kernel<<<1, 1024, smem, stream>>>(labels, n, nc, order, start, sizes, gcur, use_smem);
    OTIF_LAUNCH_CHECK();
    member_gather_kernel<<<sms * 8, 256, 0, stream>>>(P, order, start, nc, 2 * npts, Pm);
    OTIF_LAUNCH_CHECK();
    const size_t csmem = (size_t)kCenterStages * kCenterRows * 2 * npts * 4;
    if (csmem > 48 * 1024)
        OTIF_CUDA(cudaFuncSetAttribute(centers_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)csmem));
    centers_kernel<<<(unsigned)nc, 32, csmem, stream>>>(Pm, start, npts, nc, centers);
    OTIF_LAUNCH_CHECK();
    return OTIF_OK;
}

extern "C" otif_status otif_track_refine(const float *pts, const int64_t *offsets, int64_t m, int32_t npts,
                                         const float *centers, const int32_t *sizes, int32_t nc, int32_t k, float rho,
                                         float *out, int32_t *used, cudaStream_t stream) {
    OTIF_REQUIRE(m >= 0 && nc >= 0 && npts >= 2 && npts <= kMaxPts && k >= 1 && k <= kMaxK,
                 "otif_track_refine: m=%lld nc=%d npts=%d k=%d (1..%d)", (long long)m, nc, npts, k, kMaxK);
    if (m == 0) return OTIF_OK;
    OTIF_REQUIRE(pts && offsets && out && used && (nc == 0 || (centers && sizes)), "otif_track_refine: NULL argument");
    OTIF_REQUIRE(aligned8(pts), "otif_track_refine: pts must be 8-byte aligned");
    const size_t smem = (size_t)nc * center_pitch(npts) * 4 + (size_t)((nc + 1) & ~1) * 4 +
                        (size_t)kRefineWarps * 32 * npts * 8;
    if (smem > 220 * 1024) {
        set_error("otif_track_refine: %d centres of %d points do not fit in shared memory", nc, npts);
        return OTIF_EUNSUPPORTED;
    }
    int sms = 0;
    otif_status st = check_device(&sms);
    if (st != OTIF_OK) return st;
    if (smem > 48 * 1024)
        OTIF_CUDA(cudaFuncSetAttribute(refine_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    int per_sm = 0;
    OTIF_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, refine_kernel, kRefineWarps * 32, smem));
    const int64_t blocks = std::min<int64_t>(cdiv(m, kRefineWarps * 32), (int64_t)sms * std::max(per_sm, 1));
    refine_kernel<<<(unsigned)blocks, kRefineWarps * 32, smem, stream>>>(reinterpret_cast<const float2 *>(pts), offsets,
                                                                        m, npts, centers, sizes, nc, k, rho, out, used);
    OTIF_LAUNCH_CHECK();
    return OTIF_OK;
}
