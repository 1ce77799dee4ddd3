// packjob.cuh — stage 5 (crop/pack) as a queue of copy units that any
// kernel's spare warps can drain.  A "pack job" describes one device batch's identity
// pack (detector resolution == source): window g of size s goes to slot[g] of batch s.
// The slot kernel (pack.cu) builds it: per size the inverse slot map (slot -> window) and
// the unit counts.  A unit is a block of R_s rows of ONE window (R_s * row bytes ~ 32 KB),
// so the destination of a unit is one contiguous, 16-B aligned range of its batch buffer
// and its source rows are one frame-row stride apart.  Units are claimed with one
// atomicAdd each, in order, by:
//   * copy warps inside the tensor-bound convolution kernels of the NEXT device batch
//     (proxy.cu: their HBM is mostly idle, so the copy traffic hides under the MMAs), and
//   * pack_units_kernel (pack.cu), which drains whatever is left.
// Every unit is copied exactly once; the bytes are the identity crop (no arithmetic), so
// the result is bit-identical to pack_kernel's.
#pragma once

#include "common.cuh"

namespace otif {

constexpr int kPackJobMaxK = 8;
constexpr uint32_t kUnitBytes = 32768;

struct PackJob {
    // static part (host-written per batch)
    const uint8_t *src;            // [n, sh, sw, 3] frames of the batch
    size_t src_bytes;
    int sh, sw, k;
    uint8_t *batch[kPackJobMaxK];  // per-size detector batches [cap_s, bh_s, bw_s, 3]
    int bw[kPackJobMaxK], bh[kPackJobMaxK];
    int rows_per_unit[kPackJobMaxK];
    int inv_off[kPackJobMaxK];     // offset of size s's slot -> window map in inv
    const otif_window *win;
    int *inv;                      // [sum_s cap_s] window index of (s, slot)
    // device part (slot kernel)
    unsigned long long units_base[kPackJobMaxK + 1];   // prefix over sizes of the unit counts
    unsigned long long next;                           // claim counter
};

// 16 bytes from an arbitrarily aligned address: two aligned 16-B loads and a funnel shift
// (byte loads within the last 32 bytes of the source allocation)
__device__ __forceinline__ uint4 pj_load16u(const uint8_t *s0, uintptr_t src_end) {
    const uintptr_t a = (uintptr_t)s0;
    const uintptr_t al = a & ~(uintptr_t)15;
    const uint32_t sh = (uint32_t)(a - al);
    if (sh == 0) return __ldcs(reinterpret_cast<const uint4 *>(al));
    if (al + 32 <= src_end) {
        const uint4 v0 = __ldcs(reinterpret_cast<const uint4 *>(al));
        const uint4 v1 = __ldcs(reinterpret_cast<const uint4 *>(al + 16));
        const uint32_t wv[8] = {v0.x, v0.y, v0.z, v0.w, v1.x, v1.y, v1.z, v1.w};
        const uint32_t q = sh >> 2, b = (sh & 3) * 8;
        uint32_t o[4];
#pragma unroll
        for (int j = 0; j < 4; j++) {
            const uint32_t lo = q == 0 ? wv[j] : q == 1 ? wv[j + 1] : q == 2 ? wv[j + 2] : wv[j + 3];
            const uint32_t hi = q == 0 ? wv[j + 1] : q == 1 ? wv[j + 2] : q == 2 ? wv[j + 3] : wv[j + 4];
            o[j] = b ? __funnelshift_r(lo, hi, b) : lo;
        }
        return make_uint4(o[0], o[1], o[2], o[3]);
    }
    uint32_t o[4];
#pragma unroll
    for (int j = 0; j < 4; j++)
        o[j] = (uint32_t)s0[4 * j] | ((uint32_t)s0[4 * j + 1] << 8) | ((uint32_t)s0[4 * j + 2] << 16) |
               ((uint32_t)s0[4 * j + 3] << 24);
    return make_uint4(o[0], o[1], o[2], o[3]);
}

// One unit, copied by a whole warp: rows [r0, r1) of window w into dst (contiguous).
// Requires row bytes % 16 == 0 (the job is only built when every size satisfies it).
// kU 16-B pieces per lane are loaded before they are stored (memory-level parallelism).
template <int kU>
__device__ __forceinline__ void pj_copy_unit(const PackJob &j, const otif_window &w, int r0, int r1, uint8_t *dst,
                                             int lane) {
    const int rb = w.w * 3;
    const int per_row = rb >> 4;
    const int n16 = (r1 - r0) * per_row;
    const size_t fstride = (size_t)j.sw * 3;
    const uint8_t *base = j.src + ((size_t)w.frame * j.sh + w.y + r0) * fstride + (size_t)w.x * 3;
    const uintptr_t src_end = (uintptr_t)j.src + j.src_bytes;
    const bool contiguous = w.x == 0 && w.w == j.sw;     // full-width rows: one byte range
    const bool aligned = ((w.x * 3) & 15) == 0 && (fstride & 15) == 0 && (((uintptr_t)j.src) & 15) == 0;
    for (int i0 = lane; i0 < n16; i0 += 32 * kU) {
        uint4 v[kU];
#pragma unroll
        for (int u = 0; u < kU; u++) {
            const int i = i0 + u * 32;
            if (i < n16) {
                const uint8_t *s;
                if (contiguous) {
                    s = base + (size_t)i * 16;
                } else {
                    const int r = i / per_row, c = i - r * per_row;
                    s = base + (size_t)r * fstride + c * 16;
                }
                v[u] = aligned ? __ldcs(reinterpret_cast<const uint4 *>(s)) : pj_load16u(s, src_end);
            }
        }
#pragma unroll
        for (int u = 0; u < kU; u++) {
            const int i = i0 + u * 32;
            if (i < n16) __stcs(reinterpret_cast<uint4 *>(dst + (size_t)i * 16), v[u]);
        }
    }
}

// Unit u of job j: its window, rows [r0, r1) and destination.
struct PjUnit {
    otif_window w;
    int r0, r1;
    uint8_t *dst;
};
__device__ __forceinline__ PjUnit pj_unit(const PackJob *j, unsigned long long u) {
    int s = 0;
    while (s + 1 < j->k && u >= j->units_base[s + 1]) s++;
    const unsigned long long t = u - j->units_base[s];
    const int rpu = j->rows_per_unit[s];
    const int upw = (j->bh[s] + rpu - 1) / rpu;          // units per window
    const int slot = (int)(t / (unsigned)upw), blk = (int)(t - (unsigned long long)slot * upw);
    const int g = j->inv[j->inv_off[s] + slot];
    PjUnit x;
    x.w = j->win[g];
    x.r0 = blk * rpu;
    x.r1 = min(x.r0 + rpu, x.w.h);
    x.dst = j->batch[s] + ((size_t)slot * j->bh[s] + x.r0) * j->bw[s] * 3;
    return x;
}

// L2 prefetch of a unit's source rows (lane i: row r0 + i, rows of 16-B aligned ranges
// only: the prefetch needs 16-B aligned addresses and sizes)
__device__ __forceinline__ void pj_prefetch_unit(const PackJob *j, const PjUnit &x, int lane) {
    const size_t fstride = (size_t)j->sw * 3;
    const uint8_t *base = j->src + ((size_t)x.w.frame * j->sh + x.w.y) * fstride + (size_t)x.w.x * 3;
    const uint32_t rb = (uint32_t)x.w.w * 3;
    if ((((uintptr_t)base) & 15) || (rb & 15) || (fstride & 15)) return;
    if (x.w.x == 0 && x.w.w == j->sw) {      // full-width rows: one contiguous range
        if (lane == 0) bulk_prefetch_l2(base + (size_t)x.r0 * fstride, (uint32_t)(x.r1 - x.r0) * rb);
        return;
    }
    for (int r = x.r0 + lane; r < x.r1; r += 32) bulk_prefetch_l2(base + (size_t)r * fstride, rb);
}

#ifndef OTIF_PJ_PREFETCH
#define OTIF_PJ_PREFETCH 0   // 1: claim one unit ahead and prefetch its rows to L2 while copying (measured slower: C2 599k vs 633k frames/s, C3 drain 7.7 vs 5.6 ms; profiles/r02y_pj_prefetch_ab.log)
#endif

// Drain units of job j with one warp until the queue is empty or *stop becomes non-zero
// (checked between units; stop may be NULL).  With OTIF_PJ_PREFETCH the warp holds one
// claimed unit in reserve whose source rows are on their way to L2 while it copies the
// current one (a reserved unit is always copied, stop or not).
template <int kU>
__device__ __forceinline__ void pj_drain_warp(PackJob *j, const volatile int *stop, int lane) {
    const unsigned long long total = j->units_base[j->k];
#if OTIF_PJ_PREFETCH
    unsigned long long u = 0;
    if (stop && *stop) return;
    if (lane == 0) u = atomicAdd(&j->next, 1ull);
    u = __shfl_sync(0xffffffffu, u, 0);
    if (u >= total) return;
    PjUnit cur = pj_unit(j, u);
    pj_prefetch_unit(j, cur, lane);
    while (true) {
        unsigned long long nu = total;
        if (!(stop && *stop)) {
            if (lane == 0) nu = atomicAdd(&j->next, 1ull);
            nu = __shfl_sync(0xffffffffu, nu, 0);
        }
        PjUnit nxt;
        if (nu < total) {
            nxt = pj_unit(j, nu);
            pj_prefetch_unit(j, nxt, lane);
        }
        pj_copy_unit<kU>(*j, cur.w, cur.r0, cur.r1, cur.dst, lane);
        if (nu >= total) return;
        cur = nxt;
    }
#else
    while (true) {
        if (stop && *stop) return;
        unsigned long long u = 0;
        if (lane == 0) u = atomicAdd(&j->next, 1ull);
        u = __shfl_sync(0xffffffffu, u, 0);
        if (u >= total) return;
        const PjUnit x = pj_unit(j, u);
        pj_copy_unit<kU>(*j, x.w, x.r0, x.r1, x.dst, lane);
    }
#endif
}

}  // namespace otif
