// resize.cu — stage 1 (reading R13): batched bilinear resize of
// u8 NHWC RGB frames, half-pixel centres, no antialias, fp32 blend, round half up.
//
// One CTA produces R consecutive output rows of one frame (a contiguous byte range
// of the NHWC output).  It stages only the DISTINCT source rows those output rows
// touch (for a 4x downscale: rows 4y+1 and 4y+2, i.e. half the source) into shared
// memory with 16-B cp.async, blends from shared memory, and writes the output
// range back with 16-B vector stores.  HBM traffic = touched source rows + output.
#include "common.cuh"

namespace otif {

constexpr int kResizeThreads = 256;
constexpr int kMaxRowsPerCta = 32;

struct ResizeGeom {
    int n, sh, sw, dh, dw, rows_per_cta, ctas_per_frame, src_row_pitch;  // pitch of a staged row (bytes, %16==0)
};

__device__ __forceinline__ void src_coord(int o, int s, int d, int &i0, int &i1, float &l) {
    // s_o = ((2o+1)s - d) / (2d), clamped at 0
    float v = (float)((2 * o + 1) * s - d) / (float)(2 * d);
    v = fmaxf(v, 0.0f);
    int a = (int)floorf(v);
    if (a > s - 1) a = s - 1;
    i0 = a;
    i1 = a + 1 < s ? a + 1 : s - 1;
    l = v - (float)a;
}

__device__ __forceinline__ void cp_async16(void *smem, const void *gmem) {
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(smem_u32(smem)), "l"(gmem) : "memory");
}

__global__ void __launch_bounds__(kResizeThreads) resize_kernel(const uint8_t *__restrict__ src,
                                                                uint8_t *__restrict__ dst, ResizeGeom g) {
    extern __shared__ __align__(16) uint8_t smem[];
    __shared__ int s_rows[2 * kMaxRowsPerCta + 2];  // distinct source rows
    __shared__ int s_y0[kMaxRowsPerCta], s_y1[kMaxRowsPerCta];
    __shared__ float s_ly[kMaxRowsPerCta];
    __shared__ int s_nrows;

    const int f = blockIdx.x / g.ctas_per_frame;
    const int ya = (blockIdx.x % g.ctas_per_frame) * g.rows_per_cta;
    const int yb = min(ya + g.rows_per_cta, g.dh);
    const int nr = yb - ya;
    const int srow_bytes = g.sw * 3;

    if (threadIdx.x == 0) {
        int cnt = 0;
        for (int y = ya; y < yb; y++) {
            int y0, y1;
            float ly;
            src_coord(y, g.sh, g.dh, y0, y1, ly);
            // rows are non-decreasing in y: dedupe against the last entries
            int s0 = -1, s1 = -1;
            for (int t = max(cnt - 2, 0); t < cnt; t++) {
                if (s_rows[t] == y0) s0 = t;
                if (s_rows[t] == y1) s1 = t;
            }
            if (s0 < 0) { s_rows[cnt] = y0; s0 = cnt++; }
            if (s1 < 0) { s_rows[cnt] = y1; s1 = cnt++; }
            s_y0[y - ya] = s0;
            s_y1[y - ya] = s1;
            s_ly[y - ya] = ly;
        }
        s_nrows = cnt;
    }
    __syncthreads();

    uint8_t *stage = smem;  // [s_nrows][src_row_pitch]
    uint8_t *outb = smem + (size_t)(2 * g.rows_per_cta + 2) * g.src_row_pitch;
    const uint8_t *fsrc = src + (size_t)f * g.sh * srow_bytes;
    const int nrows = s_nrows;
    const bool vec16 = ((srow_bytes & 15) == 0) && ((((uintptr_t)src) & 15) == 0);
    if (vec16) {
        const int per_row = srow_bytes >> 4;
        for (int i = threadIdx.x; i < nrows * per_row; i += blockDim.x) {
            int r = i / per_row, c = i - r * per_row;
            cp_async16(stage + (size_t)r * g.src_row_pitch + c * 16, fsrc + (size_t)s_rows[r] * srow_bytes + c * 16);
        }
        asm volatile("cp.async.commit_group;\ncp.async.wait_group 0;" ::: "memory");
    } else {
        for (int i = threadIdx.x; i < nrows * srow_bytes; i += blockDim.x) {
            int r = i / srow_bytes, c = i - r * srow_bytes;
            stage[(size_t)r * g.src_row_pitch + c] = fsrc[(size_t)s_rows[r] * srow_bytes + c];
        }
    }
    __syncthreads();

    // blend: one thread per output pixel
    const int npix = nr * g.dw;
    for (int e = threadIdx.x; e < npix; e += blockDim.x) {
        int yl = e / g.dw, x = e - yl * g.dw;
        int x0, x1;
        float lx;
        src_coord(x, g.sw, g.dw, x0, x1, lx);
        const float ly = s_ly[yl];
        const uint8_t *r0 = stage + (size_t)s_y0[yl] * g.src_row_pitch;
        const uint8_t *r1 = stage + (size_t)s_y1[yl] * g.src_row_pitch;
#pragma unroll
        for (int c = 0; c < 3; c++) {
            float p00 = r0[x0 * 3 + c], p01 = r0[x1 * 3 + c];
            float p10 = r1[x0 * 3 + c], p11 = r1[x1 * 3 + c];
            float v = (1.0f - ly) * ((1.0f - lx) * p00 + lx * p01) + ly * ((1.0f - lx) * p10 + lx * p11);
            float q = floorf(v + 0.5f);
            q = fminf(fmaxf(q, 0.0f), 255.0f);
            outb[e * 3 + c] = (uint8_t)q;
        }
    }
    __syncthreads();

    // store the contiguous output byte range with 16-B stores where aligned
    uint8_t *o = dst + ((size_t)f * g.dh + ya) * (size_t)g.dw * 3;
    const int len = npix * 3;
    const int head = (int)((16 - (((uintptr_t)o) & 15)) & 15);
    const int h = head < len ? head : len;
    for (int i = threadIdx.x; i < h; i += blockDim.x) o[i] = outb[i];
    const int body = (len - h) >> 4;
    if (h == 0) {  // outb is 16-B aligned: straight vector copy
        for (int i = threadIdx.x; i < body; i += blockDim.x)
            *reinterpret_cast<uint4 *>(o + i * 16) = *reinterpret_cast<const uint4 *>(outb + i * 16);
    } else {       // shared source unaligned by h bytes: assemble words
        for (int i = threadIdx.x; i < body; i += blockDim.x) {
            const uint8_t *s = outb + h + i * 16;
            uint32_t w[4];
#pragma unroll
            for (int j = 0; j < 4; j++)
                w[j] = (uint32_t)s[4 * j] | ((uint32_t)s[4 * j + 1] << 8) | ((uint32_t)s[4 * j + 2] << 16) |
                       ((uint32_t)s[4 * j + 3] << 24);
            *reinterpret_cast<uint4 *>(o + h + i * 16) = make_uint4(w[0], w[1], w[2], w[3]);
        }
    }
    for (int i = h + body * 16 + threadIdx.x; i < len; i += blockDim.x) o[i] = outb[i];
}

// Even integer downscale (sw = FX*dw, sh = fy*dh, FX in {2,4,8}, fy even): with
// half-pixel centres every output pixel is exactly the mean of the 2x2 source pixels
// (FX*x + FX/2 - 1, +1) x (fy*y + fy/2 - 1, +1) (lx = ly = 0.5), so the fp32 blend of
// the general kernel reduces exactly to (sum + 2) >> 2.  Each thread reads the 16
// source pixels (48 B, three 16-B loads) of its group of G = 16/FX output pixels on
// the two source rows, straight from global (a warp covers 1536 contiguous bytes per
// row), and writes 3G output bytes — no shared-memory staging, no per-pixel division.
template <int FX>
__device__ __forceinline__ uint32_t byte_at(const uint32_t (&w)[12], int k) {
    return (w[k >> 2] >> (8 * (k & 3))) & 0xFFu;
}

template <int FX>
__global__ void __launch_bounds__(256) resize_even_kernel(const uint8_t *__restrict__ src, uint8_t *__restrict__ dst,
                                                          int n, int sh, int sw, int dh, int dw, int fy) {
    constexpr int G = 16 / FX;  // output pixels per thread
    const int groups = dw / G;
    const int64_t total = (int64_t)n * dh * groups;
    for (int64_t idx = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; idx < total;
         idx += (int64_t)gridDim.x * blockDim.x) {
        const int g = (int)(idx % groups);
        const int64_t fr = idx / groups;
        const int y = (int)(fr % dh);
        const int f = (int)(fr / dh);
        const int r0 = fy * y + fy / 2 - 1;
        const uint8_t *row0 = src + ((size_t)f * sh + r0) * (size_t)sw * 3 + (size_t)g * 48;
        const uint8_t *row1 = row0 + (size_t)sw * 3;
        uint32_t a[12], b[12];
#pragma unroll
        for (int v = 0; v < 3; v++) {
            const uint4 x0 = __ldg(reinterpret_cast<const uint4 *>(row0) + v);
            const uint4 x1 = __ldg(reinterpret_cast<const uint4 *>(row1) + v);
            a[4 * v] = x0.x; a[4 * v + 1] = x0.y; a[4 * v + 2] = x0.z; a[4 * v + 3] = x0.w;
            b[4 * v] = x1.x; b[4 * v + 1] = x1.y; b[4 * v + 2] = x1.z; b[4 * v + 3] = x1.w;
        }
        uint32_t o[(3 * G + 3) / 4];
#pragma unroll
        for (int i = 0; i < (3 * G + 3) / 4; i++) o[i] = 0;
#pragma unroll
        for (int j = 0; j < G; j++) {
#pragma unroll
            for (int c = 0; c < 3; c++) {
                const int k0 = (FX * j + FX / 2 - 1) * 3 + c, k1 = k0 + 3;
                const uint32_t s = byte_at<FX>(a, k0) + byte_at<FX>(a, k1) + byte_at<FX>(b, k0) + byte_at<FX>(b, k1);
                const int ob = 3 * j + c;
                o[ob >> 2] |= ((s + 2) >> 2) << (8 * (ob & 3));
            }
        }
        uint8_t *out = dst + (((size_t)f * dh + y) * dw + (size_t)g * G) * 3;
        if constexpr (G == 8) {         // 24 B, 8-B aligned
#pragma unroll
            for (int i = 0; i < 3; i++)
                reinterpret_cast<uint2 *>(out)[i] = make_uint2(o[2 * i], o[2 * i + 1]);
        } else if constexpr (G == 4) {  // 12 B, 4-B aligned
#pragma unroll
            for (int i = 0; i < 3; i++) reinterpret_cast<uint32_t *>(out)[i] = o[i];
        } else {                        // 6 B, 2-B aligned
            reinterpret_cast<uint16_t *>(out)[0] = (uint16_t)o[0];
            reinterpret_cast<uint16_t *>(out)[1] = (uint16_t)(o[0] >> 16);
            reinterpret_cast<uint16_t *>(out)[2] = (uint16_t)o[1];
        }
    }
}

otif_status launch_resize(const uint8_t *src, int32_t n, int32_t sh, int32_t sw, uint8_t *dst, int32_t dh,
                          int32_t dw, cudaStream_t stream) {
    if (n == 0) return OTIF_OK;
    {
        const int fx = sw % dw == 0 ? sw / dw : 0, fy = sh % dh == 0 ? sh / dh : 0;
        if ((fx == 2 || fx == 4 || fx == 8) && fy >= 2 && fy % 2 == 0 && dw % (16 / fx) == 0 &&
            (((uintptr_t)src) & 15) == 0 && (((uintptr_t)dst) & 7) == 0) {
            int num_sms = 148;
            check_device(&num_sms);
            const int64_t total = (int64_t)n * dh * (dw / (16 / fx));
            int64_t blocks = cdiv(total, 256);
            if (blocks > (int64_t)num_sms * 32) blocks = (int64_t)num_sms * 32;
            if (fx == 2) resize_even_kernel<2><<<(unsigned)blocks, 256, 0, stream>>>(src, dst, n, sh, sw, dh, dw, fy);
            else if (fx == 4) resize_even_kernel<4><<<(unsigned)blocks, 256, 0, stream>>>(src, dst, n, sh, sw, dh, dw, fy);
            else resize_even_kernel<8><<<(unsigned)blocks, 256, 0, stream>>>(src, dst, n, sh, sw, dh, dw, fy);
            OTIF_LAUNCH_CHECK();
            return OTIF_OK;
        }
    }
    ResizeGeom g;
    g.n = n; g.sh = sh; g.sw = sw; g.dh = dh; g.dw = dw;
    g.src_row_pitch = (int)round_up((int64_t)sw * 3, 16);
    // ~40 KB of staged source rows + output rows per CTA: several CTAs per SM overlap
    // one CTA's loads with another's blend
    const int64_t budget = 40 * 1024;
    int R = (int)(budget / (2 * g.src_row_pitch + (int64_t)dw * 3));
    R = R < 1 ? 1 : (R > kMaxRowsPerCta ? kMaxRowsPerCta : R);
    R = R > dh ? dh : R;
    g.rows_per_cta = R;
    g.ctas_per_frame = (int)cdiv(dh, R);
    size_t smem = (size_t)(2 * R + 2) * g.src_row_pitch + (size_t)R * dw * 3 + 16;
    if (smem > 200 * 1024) {
        set_error("otif_resize: source rows of %d px do not fit the staging buffer", sw);
        return OTIF_EUNSUPPORTED;
    }
    OTIF_CUDA(cudaFuncSetAttribute(resize_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    int64_t grid = (int64_t)n * g.ctas_per_frame;
    if (grid > 0x7FFFFFFF) {
        set_error("otif_resize: batch too large");
        return OTIF_EINVAL;
    }
    resize_kernel<<<(unsigned)grid, kResizeThreads, smem, stream>>>(src, dst, g);
    OTIF_LAUNCH_CHECK();
    return OTIF_OK;
}

}  // namespace otif

extern "C" otif_status otif_resize(const uint8_t *src, int32_t n, int32_t src_h, int32_t src_w, uint8_t *dst,
                                   int32_t dst_h, int32_t dst_w, cudaStream_t stream) {
    OTIF_REQUIRE(n >= 0 && src_h > 0 && src_w > 0 && dst_h > 0 && dst_w > 0,
                 "otif_resize: sizes must be positive (n=%d src=%dx%d dst=%dx%d)", n, src_w, src_h, dst_w, dst_h);
    OTIF_REQUIRE(n == 0 || (src && dst), "otif_resize: NULL pointer");
    otif_status st = otif::check_device(nullptr);
    if (st != OTIF_OK) return st;
    return otif::launch_resize(src, n, src_h, src_w, dst, dst_h, dst_w, stream);
}
