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

// Drain units of job j with one warp until the queue is empty or *stop becomes non-zero
// (checked between units; stop may be NULL).
template <int kU>
__device__ __forceinline__ void pj_drain_warp(PackJob *j, const volatile int *stop, int lane) {
    const unsigned long long total = j->units_base[j->k];
    while (true) {
        if (stop && *stop) return;
        unsigned long long u = 0;
        if (lane == 0) u = atomicAdd(&j->next, 1ull);
        u = __shfl_sync(0xffffffffu, u, 0);
        if (u >= total) return;
        int s = 0;
        while (s + 1 < j->k && u >= j->units_base[s + 1]) s++;
        const unsigned long long t = u - j->units_base[s];
        const int rpu = j->rows_per_unit[s];
        const int upw = (j->bh[s] + rpu - 1) / rpu;          // units per window
        const int slot = (int)(t / (unsigned)upw), blk = (int)(t - (unsigned long long)slot * upw);
        const int g = j->inv[j->inv_off[s] + slot];
        const otif_window w = j->win[g];
        const int r0 = blk * rpu, r1 = min(r0 + rpu, w.h);
        uint8_t *dst = j->batch[s] + ((size_t)slot * j->bh[s] + r0) * j->bw[s] * 3;
        pj_copy_unit<kU>(*j, w, r0, r1, dst, lane);
    }
}

}  // namespace otif
