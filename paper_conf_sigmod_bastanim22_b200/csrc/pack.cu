// pack.cu — stage 5: crop (and, when the detector resolution differs
// from the source, bilinearly resample) every window into its per-size dense
// detector batch.  Slot = running count of the window's size in emission order.
//
// K7a slot_kernel: one CTA scans the window list in order; per size, a warp ballot
//   gives each window its rank among same-size windows of its 32-window group, and
//   running per-size carries make the slot.  size_count is written at the end.
// K7b pack_kernel: persistent grid; one CTA per window (grid-stride).  Identity case:
//   each thread produces 16 destination bytes (destination rows are 16-B aligned for
//   every size in W with w*3 % 16 == 0) from two aligned 16-B source loads and a
//   funnel shift, since a window's x offset makes the source row arbitrarily aligned.
//   Resampling case: per output pixel bilinear blend (same arithmetic as resize.cu).
#include <stddef.h>
#include <string.h>

#include "common.cuh"
#include "packjob.cuh"

namespace otif {

constexpr int kMaxK = 8;

struct PackParams {
    const uint8_t *src;
    int n, sh, sw, dh, dw;
    size_t src_bytes;
    const otif_window *win;
    const int *total;
    int capacity;
    int k;
    uint8_t *batch[kMaxK];
    int cap[kMaxK];
    int bw[kMaxK], bh[kMaxK];
    int *slot;
    int *size_count;
    unsigned long long *ctr_pack;  // internal (pipeline): [0] windows dropped for batch_cap, [1] packed pixels
    int stage_bytes;  // bulk ring stage size (<= kBulkStage)
    PackJob *job;     // internal (pipeline): build the copy-unit queue (packjob.cuh) instead of copying here
};

__global__ void __launch_bounds__(1024) slot_kernel(const __grid_constant__ PackParams p) {
    __shared__ int s_warp_cnt[32][kMaxK];
    __shared__ int s_carry[kMaxK];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nw = blockDim.x >> 5;
    if (threadIdx.x < kMaxK) s_carry[threadIdx.x] = 0;
    __syncthreads();
    const int total = min(*p.total, p.capacity);
    unsigned long long dropped = 0, packed_px = 0;
    for (int base = 0; base < total; base += blockDim.x) {
        const int g = base + threadIdx.x;
        const int s = g < total ? p.win[g].size_idx : -1;
        int rank = 0;
        for (int z = 0; z < p.k; z++) {
            unsigned m = __ballot_sync(0xffffffffu, s == z);
            if (s == z) rank = __popc(m & ((1u << lane) - 1u));
            if (lane == 0) s_warp_cnt[warp][z] = __popc(m);
        }
        __syncthreads();
        if (g < total) {
            int pre = s_carry[s];
            for (int w = 0; w < warp; w++) pre += s_warp_cnt[w][s];
            p.slot[g] = pre + rank;
            if (pre + rank < p.cap[s]) {
                packed_px += (unsigned long long)p.win[g].w * p.win[g].h;
                if (p.job) p.job->inv[p.job->inv_off[s] + pre + rank] = g;
            } else {
                dropped++;
            }
        }
        __syncthreads();
        if (threadIdx.x < p.k) {
            int add = 0;
            for (int w = 0; w < nw; w++) add += s_warp_cnt[w][threadIdx.x];
            s_carry[threadIdx.x] += add;
        }
        __syncthreads();
    }
    // size_count counts every listed window, including those dropped for batch_cap
    if (threadIdx.x < p.k) p.size_count[threadIdx.x] = s_carry[threadIdx.x];
    if (p.job && threadIdx.x == 0) {
        // unit queue: per size min(count, cap) windows x ceil(h / rows_per_unit) units
        unsigned long long base = 0;
        for (int z = 0; z < p.k; z++) {
            p.job->units_base[z] = base;
            const int kept = min(s_carry[z], p.cap[z]);
            const int rpu = p.job->rows_per_unit[z];
            base += (unsigned long long)kept * ((p.bh[z] + rpu - 1) / rpu);
        }
        for (int z = p.k; z <= kPackJobMaxK; z++) p.job->units_base[z] = base;
        p.job->next = 0;
    }
    if (p.ctr_pack) {
        for (int o = 16; o > 0; o >>= 1) {
            dropped += __shfl_xor_sync(0xffffffffu, dropped, o);
            packed_px += __shfl_xor_sync(0xffffffffu, packed_px, o);
        }
        if (lane == 0 && (dropped | packed_px)) {
            atomicAdd(&p.ctr_pack[0], dropped);
            atomicAdd(&p.ctr_pack[1], packed_px);
        }
    }
}

__device__ __forceinline__ uint32_t fshift(uint32_t lo, uint32_t hi, uint32_t sh_bytes) {
    return sh_bytes ? __funnelshift_r(lo, hi, sh_bytes * 8) : lo;
}

// 16 bytes from an arbitrarily aligned address: two aligned 16-B loads and a funnel shift
// (byte loads only within the last 32 bytes of the source allocation)
__device__ __forceinline__ uint4 load16u(const uint8_t *s0, uintptr_t src_end) {
    const uintptr_t a = (uintptr_t)s0;
    const uintptr_t al = a & ~(uintptr_t)15;
    const uint32_t sh = (uint32_t)(a - al);
    if (al + 32 <= src_end) {
        const uint4 v0 = __ldg(reinterpret_cast<const uint4 *>(al));
        if (sh == 0) return v0;
        const uint4 v1 = __ldg(reinterpret_cast<const uint4 *>(al + 16));
        const uint32_t wv[8] = {v0.x, v0.y, v0.z, v0.w, v1.x, v1.y, v1.z, v1.w};
        const uint32_t q = sh >> 2, b = sh & 3;
        uint32_t o[4];
#pragma unroll
        for (int j = 0; j < 4; j++) {
            // wv[q + j], wv[q + j + 1] with q in 0..3 (unrolled select, no local memory)
            uint32_t lo = q == 0 ? wv[j] : q == 1 ? wv[j + 1] : q == 2 ? wv[j + 2] : wv[j + 3];
            uint32_t hi = q == 0 ? wv[j + 1] : q == 1 ? wv[j + 2] : q == 2 ? wv[j + 3] : wv[j + 4];
            o[j] = fshift(lo, hi, b);
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

// TMA bulk path for windows whose source rows are 16-B aligned (all windows placed on
// 16-px multiples, which the cell grid produces for most of them): one thread streams
// the window through a ring of shared-memory chunks with 1-D bulk async copies —
// global->shared (the window's rows of a chunk; a single copy when the window spans
// full frame rows, so its bytes are contiguous) then shared->global into the packed
// detector batch (contiguous).  Loads run kBulkLead chunks ahead of the stores.
// STAGES ring stages, loads run STAGES - 2 chunks ahead of the stores (one stage is being
// read by an in-flight store); stage size is a launch parameter (<= kBulkStage).
constexpr int kBulkStage = 16384;            // ring stage (bytes)
constexpr int kPackStages = 3;

__device__ __forceinline__ void bulk_s2g(void *dst_gmem, const void *src_smem, uint32_t bytes) {
    asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(dst_gmem), "r"(smem_u32(src_smem)),
                 "r"(bytes)
                 : "memory");
}
__device__ __forceinline__ void bulk_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void bulk_wait_read() {
    asm volatile("cp.async.bulk.wait_group.read %0;" ::"n"(N) : "memory");
}
__device__ __forceinline__ void bulk_wait_all() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }

// One thread streams one window through the ring.  A window spanning full frame rows is
// one contiguous byte range in the source: it moves in 16 KB chunks regardless of rows;
// otherwise a chunk is as many whole rows as fit in a stage (one g2s per row).
template <int kBulkStages>
__device__ void pack_window_bulk(uint8_t *ring, uint64_t *bars, uint32_t &chunk_seq, const uint8_t *fbase, int sw,
                                 const otif_window &w, uint8_t *dst, uint32_t stage_bytes) {
    constexpr int kBulkLead = kBulkStages - 2;
    const uint32_t row_bytes = (uint32_t)w.w * 3;
    const bool contiguous = (w.x == 0 && w.w == sw);
    const uint32_t total = (uint32_t)w.h * row_bytes;
    const int rpc = (int)(stage_bytes / row_bytes);  // >= 1 (checked by the caller)
    const uint32_t chunk_bytes = contiguous ? stage_bytes : rpc * row_bytes;
    const int nchunks = (int)((total + chunk_bytes - 1) / chunk_bytes);
    const uint8_t *wsrc = fbase + ((size_t)w.y * sw + w.x) * 3;
    const uint32_t base = chunk_seq;
    for (int i = 0; i < nchunks + kBulkLead; i++) {
        if (i < nchunks) {
            const uint32_t c = base + i, s = c % kBulkStages;
            // stage s is reused by chunk i: the store of chunk i - kBulkStages must have read it
            bulk_wait_read<kBulkStages - kBulkLead - 1>();
            const uint32_t off = (uint32_t)i * chunk_bytes;
            const uint32_t bytes = min(chunk_bytes, total - off);
            uint8_t *buf = ring + (size_t)s * stage_bytes;
            mbar_arrive_expect_tx(&bars[s], bytes);
            if (contiguous) {
                bulk_g2s(buf, wsrc + off, bytes, &bars[s]);
            } else {
                const int r0 = i * rpc, nr = (int)(bytes / row_bytes);
                for (int r = 0; r < nr; r++)
                    bulk_g2s(buf + r * row_bytes, wsrc + (size_t)(r0 + r) * sw * 3, row_bytes, &bars[s]);
            }
        }
        const int j = i - kBulkLead;
        if (j >= 0 && j < nchunks) {
            const uint32_t c = base + j, s = c % kBulkStages;
            mbar_wait(&bars[s], (c / kBulkStages) & 1);
            const uint32_t off = (uint32_t)j * chunk_bytes;
            bulk_s2g(dst + off, ring + (size_t)s * stage_bytes, min(chunk_bytes, total - off));
            bulk_commit();
        }
    }
    chunk_seq = base + nchunks;
    bulk_wait_all();
}

template <int kBulkStages, int kThreads>
__global__ void __launch_bounds__(kThreads) pack_kernel(const __grid_constant__ PackParams p) {
    extern __shared__ __align__(128) uint8_t ring[];  // kBulkStages x p.stage_bytes
    __shared__ uint64_t bars[kBulkStages];
    if (threadIdx.x == 0) {
        for (int i = 0; i < kBulkStages; i++) mbar_init(&bars[i], 1);
        fence_barrier_init();
    }
    __syncthreads();
    uint32_t chunk_seq = 0;
    const int total = min(*p.total, p.capacity);
    const bool identity = (p.dh == p.sh && p.dw == p.sw);
    for (int g = blockIdx.x; g < total; g += gridDim.x) {
        const otif_window w = p.win[g];
        const int s = w.size_idx;
        const int sl = p.slot[g];
        if (sl >= p.cap[s]) continue;
        uint8_t *dst = p.batch[s] + (size_t)sl * p.bh[s] * p.bw[s] * 3;
        const int row_bytes = w.w * 3;
        if (identity && (row_bytes & 15) == 0 && row_bytes <= p.stage_bytes && (((uintptr_t)p.batch[s]) & 15) == 0 &&
            ((w.x * 3) & 15) == 0 && ((p.sw * 3) & 15) == 0 && (((uintptr_t)p.src) & 15) == 0) {
            if (threadIdx.x == 0)
                pack_window_bulk<kBulkStages>(ring, bars, chunk_seq, p.src + (size_t)w.frame * p.sh * p.sw * 3, p.sw, w,
                                              dst, (uint32_t)p.stage_bytes);
        } else if (identity && (row_bytes & 15) == 0 && (((uintptr_t)p.batch[s]) & 15) == 0) {
            const int per_row = row_bytes >> 4;
            const uint8_t *fbase = p.src + (size_t)w.frame * p.sh * p.sw * 3;
            const uintptr_t src_end = (uintptr_t)p.src + p.src_bytes;
            const int total16 = w.h * per_row;
            // 4 independent 16-B loads in flight per thread before the stores (memory-level parallelism)
            for (int i0 = threadIdx.x; i0 < total16; i0 += 4 * blockDim.x) {
                uint4 v[4];
#pragma unroll
                for (int u = 0; u < 4; u++) {
                    const int i = i0 + u * blockDim.x;
                    if (i < total16) {
                        const int r = i / per_row, c = i - r * per_row;
                        v[u] = load16u(fbase + ((size_t)(w.y + r) * p.sw + w.x) * 3 + c * 16, src_end);
                    }
                }
#pragma unroll
                for (int u = 0; u < 4; u++) {
                    const int i = i0 + u * blockDim.x;
                    if (i < total16) {
                        const int r = i / per_row, c = i - r * per_row;
                        *reinterpret_cast<uint4 *>(dst + (size_t)r * row_bytes + c * 16) = v[u];
                    }
                }
            }
        } else if (identity) {
            const uint8_t *fbase = p.src + (size_t)w.frame * p.sh * p.sw * 3;
            for (int i = threadIdx.x; i < w.h * row_bytes; i += blockDim.x) {
                const int r = i / row_bytes, c = i - r * row_bytes;
                dst[(size_t)r * row_bytes + c] = fbase[((size_t)(w.y + r) * p.sw + w.x) * 3 + c];
            }
        } else {
            // resample: det pixel (w.y + r, w.x + x) of the det_h x det_w frame, bilinear from src
            const uint8_t *fbase = p.src + (size_t)w.frame * p.sh * p.sw * 3;
            for (int i = threadIdx.x; i < w.h * w.w; i += blockDim.x) {
                const int r = i / w.w, x = i - r * w.w;
                const int oy = w.y + r, ox = w.x + x;
                float sy = fmaxf((float)((2 * oy + 1) * p.sh - p.dh) / (float)(2 * p.dh), 0.0f);
                float sx = fmaxf((float)((2 * ox + 1) * p.sw - p.dw) / (float)(2 * p.dw), 0.0f);
                int y0 = min((int)floorf(sy), p.sh - 1), x0 = min((int)floorf(sx), p.sw - 1);
                int y1 = min(y0 + 1, p.sh - 1), x1 = min(x0 + 1, p.sw - 1);
                float ly = sy - (float)y0, lx = sx - (float)x0;
#pragma unroll
                for (int c = 0; c < 3; c++) {
                    float p00 = fbase[((size_t)y0 * p.sw + x0) * 3 + c], p01 = fbase[((size_t)y0 * p.sw + x1) * 3 + c];
                    float p10 = fbase[((size_t)y1 * p.sw + x0) * 3 + c], p11 = fbase[((size_t)y1 * p.sw + x1) * 3 + c];
                    float v = (1.0f - ly) * ((1.0f - lx) * p00 + lx * p01) + ly * ((1.0f - lx) * p10 + lx * p11);
                    v = fminf(fmaxf(floorf(v + 0.5f), 0.0f), 255.0f);
                    dst[(size_t)i * 3 + c] = (uint8_t)v;
                }
            }
        }
    }
}

// Drains a pack job's remaining copy units (those the fused copy warps of the proxy did
// not take): 4 warps per CTA, several CTAs per SM.
__global__ void __launch_bounds__(128) pack_units_kernel(PackJob *job) {
    pj_drain_warp<8>(job, nullptr, threadIdx.x & 31);
}

}  // namespace otif

using namespace otif;

namespace otif {

// A pack job applies when the detector resolution is the source's (identity crop) and every
// size's rows are whole 16-B pieces (w * 3 % 16 == 0) in 16-B aligned batch buffers.
bool pack_job_applies(int32_t src_h, int32_t src_w, int32_t det_h, int32_t det_w, const otif_wsize *sizes, int32_t k,
                      uint8_t *const *batches) {
    if (src_h != det_h || src_w != det_w || k > kPackJobMaxK) return false;
    for (int s = 0; s < k; s++)
        if ((sizes[s].w * 3) % 16 != 0 || (((uintptr_t)batches[s]) & 15) != 0) return false;
    return true;
}

// Stage-5 slot assignment that also builds the copy-unit queue `job_dev` (device) for
// later draining (fused copy warps, pack_units_kernel).  inv: >= sum(batch_cap) ints.
otif_status launch_pack_prepare(const uint8_t *src, int32_t n, int32_t src_h, int32_t src_w,
                                const otif_window *windows, const int32_t *total, int32_t capacity,
                                const otif_wsize *sizes, int32_t k, uint8_t *const *batches, const int32_t *batch_cap,
                                int32_t *slot, int32_t *size_count, cudaStream_t stream, unsigned long long *ctr_pack,
                                PackJob *job_dev, int *inv) {
    PackJob h;
    memset(&h, 0, sizeof(h));
    h.src = src; h.src_bytes = (size_t)n * src_h * src_w * 3; h.sh = src_h; h.sw = src_w; h.k = k;
    h.win = windows; h.inv = inv;
    int off = 0;
    for (int s = 0; s < k; s++) {
        h.batch[s] = batches[s]; h.bw[s] = sizes[s].w; h.bh[s] = sizes[s].h;
        const int rb = sizes[s].w * 3;
        int rpu = (int)(kUnitBytes / (uint32_t)rb);
        h.rows_per_unit[s] = rpu < 1 ? 1 : (rpu > sizes[s].h ? sizes[s].h : rpu);
        h.inv_off[s] = off;
        off += batch_cap[s];
    }
    // static part; the slot kernel fills units_base / next (stream order)
    OTIF_CUDA(cudaMemcpyAsync(job_dev, &h, offsetof(PackJob, units_base), cudaMemcpyHostToDevice, stream));
    PackParams p;
    memset(&p, 0, sizeof(p));
    p.src = src; p.n = n; p.sh = src_h; p.sw = src_w; p.dh = src_h; p.dw = src_w;
    p.win = windows; p.total = total; p.capacity = capacity; p.k = k;
    for (int s = 0; s < k; s++) {
        p.batch[s] = batches[s]; p.cap[s] = batch_cap[s]; p.bw[s] = sizes[s].w; p.bh[s] = sizes[s].h;
    }
    p.slot = slot; p.size_count = size_count; p.ctr_pack = ctr_pack; p.job = job_dev;
    slot_kernel<<<1, 1024, 0, stream>>>(p);
    OTIF_LAUNCH_CHECK();
    return OTIF_OK;
}

otif_status launch_pack_units(PackJob *job_dev, cudaStream_t stream) {
    int num_sms = 148;
    check_device(&num_sms);
    pack_units_kernel<<<num_sms * 8, 128, 0, stream>>>(job_dev);
    OTIF_LAUNCH_CHECK();
    return OTIF_OK;
}

// internal entry; ctr_pack (pipeline, may be NULL): device counters of dropped windows
// and packed pixels, accumulated
otif_status launch_pack(const uint8_t *src, int32_t n, int32_t src_h, int32_t src_w, int32_t det_h, int32_t det_w,
                        const otif_window *windows, const int32_t *total, int32_t capacity, const otif_wsize *sizes,
                        int32_t k, uint8_t *const *batches, const int32_t *batch_cap, int32_t *slot,
                        int32_t *size_count, cudaStream_t stream, unsigned long long *ctr_pack) {
    PackParams p;
    memset(&p, 0, sizeof(p));
    p.src = src; p.n = n; p.sh = src_h; p.sw = src_w; p.dh = det_h; p.dw = det_w;
    p.src_bytes = (size_t)n * src_h * src_w * 3;
    p.win = windows; p.total = total; p.capacity = capacity; p.k = k;
    for (int s = 0; s < k; s++) {
        OTIF_REQUIRE(sizes[s].w > 0 && sizes[s].h > 0 && sizes[s].w <= det_w && sizes[s].h <= det_h,
                     "otif_pack_windows: size %d larger than the detector frame", s);
        OTIF_REQUIRE(batch_cap[s] >= 0 && (batch_cap[s] == 0 || batches[s]), "otif_pack_windows: batch %d", s);
        p.batch[s] = batches[s]; p.cap[s] = batch_cap[s]; p.bw[s] = sizes[s].w; p.bh[s] = sizes[s].h;
    }
    p.slot = slot; p.size_count = size_count;
    p.ctr_pack = ctr_pack;
    p.stage_bytes = kBulkStage;
    int num_sms = 148;
    check_device(&num_sms);
    slot_kernel<<<1, 1024, 0, stream>>>(p);
    OTIF_LAUNCH_CHECK();
    if (capacity > 0) {
        // persistent grid: 6 CTAs per SM (3 x 16 KB rings each), one window per CTA at a time
        const int want = num_sms * 6;
        const int grid = capacity < want ? capacity : want;
        const int smem = kPackStages * p.stage_bytes;
        auto kern = pack_kernel<kPackStages, 128>;
        OTIF_CUDA(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
        kern<<<grid, 128, smem, stream>>>(p);
        OTIF_LAUNCH_CHECK();
    }
    return OTIF_OK;
}

}  // namespace otif

extern "C" otif_status otif_pack_windows(const uint8_t *src, int32_t n, int32_t src_h, int32_t src_w, int32_t det_h,
                                         int32_t det_w, const otif_window *windows, const int32_t *total,
                                         int32_t capacity, const otif_wsize *sizes, int32_t k,
                                         uint8_t *const *batches, const int32_t *batch_cap, int32_t *slot,
                                         int32_t *size_count, cudaStream_t stream) {
    OTIF_REQUIRE(n >= 0 && src_h > 0 && src_w > 0 && det_h > 0 && det_w > 0, "otif_pack_windows: bad sizes");
    OTIF_REQUIRE(k >= 1 && k <= kMaxK, "otif_pack_windows: k=%d not in [1,8]", k);
    OTIF_REQUIRE(sizes && batches && batch_cap, "otif_pack_windows: NULL host arrays");
    OTIF_REQUIRE(total && size_count && capacity >= 0, "otif_pack_windows: NULL total/size_count");
    OTIF_REQUIRE(capacity == 0 || (windows && slot), "otif_pack_windows: NULL windows/slot");
    OTIF_REQUIRE(src || n == 0, "otif_pack_windows: NULL src");
    otif_status st = check_device(nullptr);
    if (st != OTIF_OK) return st;
    return launch_pack(src, n, src_h, src_w, det_h, det_w, windows, total, capacity, sizes, k, batches, batch_cap,
                       slot, size_count, stream, nullptr);
}
