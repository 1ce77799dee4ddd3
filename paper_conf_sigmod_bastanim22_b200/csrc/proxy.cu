// proxy.cu — stage 2: the segmentation proxy CNN (readings R1, R2, R4).
//
//   E1 (3->32, 3x3, stride 2): tcgen05 M=128,N=32 tiles with K = 27 padded to 32;
//       the A rows are gathered from the u8 proxy image by the CTA's threads.
//   E2..E5, D1 (3x3, pad 1): implicit-GEMM convolutions on the 5th-gen tensor cores
//       (tcgen05.mma kind::f16, bf16 x bf16 -> fp32 in TMEM), one persistent,
//       warp-specialised kernel per layer.
//   D2 (1x1, 128->1) + sigmoid: fused into D1's epilogue (per-row GEMV over the
//       bf16-rounded D1 activations read back from TMEM).
//
// Activation layout in HBM ("padded linear, chunk-planar").  A stride-1 3x3 conv over
// an H x W map reads, for output pixel q, the input pixels q + kh*(W+2) + kw of the
// zero-padded map flattened row-major with pitch W+2 — a pure linear shift per tap.
// So every GEMM layer's input is stored zero-padded and flattened, frames stacked
// (each frame owns H+1 rows of pitch W+2; the bottom pad of frame f is the top pad
// of frame f+1), and channel-chunk planar: [plane][C/8][pixels][8 bf16].  Then the
// A operand of one M tile (128 consecutive output positions) for ALL 9 taps is one
// contiguous halo of 128 + 2(W+2) + 2 pixels per 8-channel chunk, loaded once with
// 1-D bulk async copies and reused by 9 MMAs through shifted smem descriptors (the
// no-swizzle K-major layout puts consecutive rows 16 B apart, so a shift of s pixels
// is a +16*s start address).  Stride-2 layers read a parity-split input (4 planes:
// even/odd rows x even/odd cols), on which each of the 9 taps is again a linear
// shift (by 0, 1, pitch or pitch+1) within one plane.  Each layer's epilogue writes
// its output directly into the next layer's layout; pad positions are never
// written and stay zero (the workspace is zeroed once, see the tag kernels).
// Output positions in the pad columns/rows are computed and discarded (≈6–12% of
// MACs at the configs' sizes; the roofline counts only the algorithmic MACs).
#include <math.h>
#include <stdlib.h>
#include <string.h>

#include <vector>

#include "common.cuh"

namespace otif {

constexpr int kConvThreads = 256;   // warp0 producer, warp1 MMA, warp2 TMEM alloc, warps4-7 epilogue
constexpr int kTileM = 128;
constexpr int kMaxStagesA = 4;
constexpr int kMaxStagesB = 8;

// ---------------------------------------------------------------------------
// layouts
// ---------------------------------------------------------------------------
struct Layout {        // a GEMM layer's input buffer
    int kind;          // 1: stride-1 padded (1 plane); 2: parity-split (4 planes)
    int planes;
    int pitch;         // pixels per padded row
    int64_t fstride;   // pixels per frame slot
    int64_t lcap;      // pixels per (plane, chunk) row of the buffer
    int c8;            // channels / 8
    size_t offset;     // byte offset inside the workspace
    size_t bytes;
};

__host__ __device__ __forceinline__ int64_t layout_pixel(int kind, int pitch, int64_t fstride, int f, int y, int x,
                                                         int &plane) {
    if (kind == 1) {
        plane = 0;
        return (int64_t)f * fstride + (int64_t)(y + 1) * pitch + (x + 1);
    }
    plane = ((y & 1) << 1) | (x & 1);
    return (int64_t)f * fstride + (int64_t)((y >> 1) + 1) * pitch + ((x >> 1) + 1);
}

struct ConvParams {
    const uint8_t *act;         // input buffer (bytes)
    int64_t lcap;
    int c8_in;
    int kb, ncb;                // channels per K block, number of K blocks
    int P;                      // halo rows per A stage
    int ngroups;
    int group_plane[4];
    int group_ntaps[4];
    int group_shift[4][9];
    const uint8_t *wpk;         // packed bf16 weights [cb][tap-in-loop-order][chunk][N][8]
    const float *bias;          // [N]
    int N;
    int64_t mtot;
    int ntiles;
    int pitch;                  // q decode
    int64_t fstride;
    int out_h, out_w;
    int stages_a, stages_b;
    int mt;                     // 128-row sub-tiles per CTA tile (share each A halo and B stage)
    // destination
    int out_kind;               // 1/2: next layout kind; 3: head scores
    uint8_t *out;
    int64_t out_lcap;
    int out_c8;
    int out_pitch;
    int64_t out_fstride;
    float *scores;
    const float *w2;            // [N] bf16-rounded head weights (fp32 storage)
    float b2;
};

// ---------------------------------------------------------------------------
// workspace tag: zero the workspace once per layout (pads must be zero)
// ---------------------------------------------------------------------------
__global__ void ws_zero_kernel(uint8_t *ws, size_t bytes, uint64_t tag) {
    if (*reinterpret_cast<volatile uint64_t *>(ws) == tag) return;
    uint4 z = make_uint4(0, 0, 0, 0);
    size_t n16 = bytes / 16;
    for (size_t i = 16 + blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n16; i += (size_t)gridDim.x * blockDim.x)
        reinterpret_cast<uint4 *>(ws)[i] = z;
}
__global__ void ws_tag_kernel(uint8_t *ws, uint64_t tag) { *reinterpret_cast<uint64_t *>(ws) = tag; }

// ---------------------------------------------------------------------------
// E1: 3x3 stride-2 conv 3 -> 32 on the tensor cores.  K = 27 (3x3 taps x RGB) is
// padded to 32; each CTA thread gathers the 27 u8 inputs of one output pixel (its A
// row), converts them exactly to bf16 ((u-128)/128) and stores them in the no-swizzle
// K-major smem layout; one thread issues two M=128,N=32,K=16 tcgen05.mma; the same
// 128 threads read the accumulator row back (tcgen05.ld), add bias, ReLU, round to
// bf16 and store 4 x 16 B into E2's input layout.  Several CTAs per SM overlap one
// CTA's gather with another's MMA/epilogue.
// ---------------------------------------------------------------------------
struct E1Params {
    const uint8_t *img;
    int n, h, w, oh, ow;
    const uint16_t *wpk;  // [4 chunks][32 n][8] bf16, k = (kh*3+kw)*3 + c, k >= 27 zero
    const float *bias;    // [32]
    int out_kind, out_pitch;
    int64_t out_fstride, out_lcap;
    uint8_t *out;
    int64_t ntiles;
};

__global__ void __launch_bounds__(128) e1_umma_kernel(const __grid_constant__ E1Params p) {
    __shared__ __align__(128) uint8_t sA[4 * 128 * 16];  // [chunk][row][16 B]
    __shared__ __align__(128) uint8_t sB[4 * 32 * 16];   // [chunk][n][16 B]
    __shared__ float sbias[32];
    __shared__ uint64_t bar;
    __shared__ uint32_t tslot;
    const int t = threadIdx.x, warp = t >> 5;
    for (int i = t; i < 4 * 32 * 8 / 8; i += blockDim.x)
        reinterpret_cast<uint4 *>(sB)[i] = reinterpret_cast<const uint4 *>(p.wpk)[i];
    if (t < 32) sbias[t] = p.bias[t];
    if (t == 0) { mbar_init(&bar, 1); fence_barrier_init(); }
    if (warp == 0) tmem_alloc(&tslot, 32);
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem = tslot;
    const uint32_t idesc = umma_idesc_bf16(128, 32);
    uint32_t phase = 0;
    const int64_t npx = (int64_t)p.n * p.oh * p.ow;
    for (int64_t tile = blockIdx.x; tile < p.ntiles; tile += gridDim.x) {
        const int64_t px = tile * 128 + t;
        const bool valid = px < npx;
        int f = 0, oy = 0, ox = 0;
        uint32_t kv[16];
#pragma unroll
        for (int j = 0; j < 16; j++) kv[j] = 0;
        if (valid) {
            ox = (int)(px % p.ow);
            int64_t r = px / p.ow;
            oy = (int)(r % p.oh);
            f = (int)(r / p.oh);
            const uint8_t *base = p.img + (size_t)f * p.h * p.w * 3;
            float x[32];
#pragma unroll
            for (int k = 27; k < 32; k++) x[k] = 0.0f;
#pragma unroll
            for (int kh = 0; kh < 3; kh++) {
                const int iy = 2 * oy - 1 + kh;
#pragma unroll
                for (int kw = 0; kw < 3; kw++) {
                    const int ix = 2 * ox - 1 + kw;
                    const bool ok = iy >= 0 && iy < p.h && ix >= 0 && ix < p.w;
                    const uint8_t *q = base + ((ptrdiff_t)iy * p.w + ix) * 3;
#pragma unroll
                    for (int c = 0; c < 3; c++)
                        x[(kh * 3 + kw) * 3 + c] = ok ? (float)((int)__ldg(q + c) - 128) * 0.0078125f : 0.0f;
                }
            }
#pragma unroll
            for (int j = 0; j < 16; j++) kv[j] = pack_bf16x2(x[2 * j], x[2 * j + 1]);  // exact
        }
#pragma unroll
        for (int c = 0; c < 4; c++)
            *reinterpret_cast<uint4 *>(sA + (c * 128 + t) * 16) = make_uint4(kv[4 * c], kv[4 * c + 1], kv[4 * c + 2], kv[4 * c + 3]);
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");  // generic-proxy stores -> tensor core
        tc_fence_before();
        __syncthreads();
        if (t == 0) {
            tc_fence_after();
            const uint32_t a0 = smem_u32(sA), b0 = smem_u32(sB);
#pragma unroll
            for (int s = 0; s < 2; s++)
                umma_bf16(tmem, umma_desc(a0 + 2 * s * 2048, 2048, 128), umma_desc(b0 + 2 * s * 512, 512, 128), idesc, s);
            umma_commit(&bar);
        }
        mbar_wait(&bar, phase);
        phase ^= 1;
        tc_fence_after();
        uint32_t v[32];
        tmem_ld32(tmem + ((uint32_t)(warp * 32) << 16), v);
        if (valid) {
            int plane;
            const int64_t L = layout_pixel(p.out_kind, p.out_pitch, p.out_fstride, f, oy, ox, plane);
#pragma unroll
            for (int cc = 0; cc < 4; cc++) {
                uint32_t pk[4];
#pragma unroll
                for (int j = 0; j < 4; j++) {
                    float a0 = fmaxf(__uint_as_float(v[cc * 8 + 2 * j]) + sbias[cc * 8 + 2 * j], 0.0f);
                    float a1 = fmaxf(__uint_as_float(v[cc * 8 + 2 * j + 1]) + sbias[cc * 8 + 2 * j + 1], 0.0f);
                    pk[j] = pack_bf16x2(a0, a1);
                }
                *reinterpret_cast<uint4 *>(p.out + (((size_t)plane * 4 + cc) * p.out_lcap + L) * 16) =
                    make_uint4(pk[0], pk[1], pk[2], pk[3]);
            }
        }
        tc_fence_before();
        __syncthreads();  // accumulator read and smem A consumed before the next tile overwrites them
    }
    tc_fence_after();
    if (warp == 0) tmem_dealloc(tmem, 32);
}

// ---------------------------------------------------------------------------
// E2..E5, D1: persistent warp-specialised implicit-GEMM conv on tcgen05
// ---------------------------------------------------------------------------
// SWAP (head layer, N = 128, MT = 2): the operands trade places — the weights are the
// M = 128 operand and the 256 halo rows the N = 256 operand — so one M128 x N256 MMA
// reads 12 KB of shared memory per 1 MFLOP instead of two M128 x N128 MMAs reading 16 KB
// (N = 128 layers are shared-memory-bandwidth bound).  The accumulator is transposed
// (TMEM lane = output channel, column = pixel); the head epilogue reduces the D2 dot
// product across lanes (reduce-scatter shuffles) and across the 4 epilogue warps.
template <int MT, bool SWAP = false>
__global__ void __launch_bounds__(kConvThreads, 1) conv_umma_kernel(const __grid_constant__ ConvParams p) {
    extern __shared__ __align__(1024) uint8_t smem[];
    const int warp = threadIdx.x >> 5;
    const int lane = threadIdx.x & 31;

    const uint32_t chunks = p.kb >> 3;
    const uint32_t a_bytes = chunks * p.P * 16;
    const uint32_t b_bytes = (uint32_t)p.N * p.kb * 2;
    uint8_t *a_buf = smem;
    uint8_t *b_buf = a_buf + (size_t)p.stages_a * a_bytes;
    uint64_t *bars = reinterpret_cast<uint64_t *>(b_buf + (size_t)p.stages_b * b_bytes);
    uint64_t *a_full = bars;
    uint64_t *a_empty = a_full + kMaxStagesA;
    uint64_t *b_full = a_empty + kMaxStagesA;
    uint64_t *b_empty = b_full + kMaxStagesB;
    uint64_t *t_full = b_empty + kMaxStagesB;   // 2 accumulator stages
    uint64_t *t_empty = t_full + 2;
    uint32_t *tmem_slot = reinterpret_cast<uint32_t *>(t_empty + 2);
    float *s_bias = reinterpret_cast<float *>(tmem_slot + 4);
    float *s_w2 = s_bias + 256;
    float *s_red = s_w2 + 256;               // SWAP head: [4 warps][256 pixels] partial dots

    const uint32_t acc_cols = 2 * MT * p.N;  // two accumulator stages of MT sub-tiles x N columns
    const uint32_t tmem_cols = acc_cols <= 32 ? 32 : (acc_cols <= 64 ? 64 : (acc_cols <= 128 ? 128 : (acc_cols <= 256 ? 256 : 512)));

    if (threadIdx.x == 0) {
        for (int i = 0; i < p.stages_a; i++) { mbar_init(&a_full[i], 1); mbar_init(&a_empty[i], 1); }
        for (int i = 0; i < p.stages_b; i++) { mbar_init(&b_full[i], 1); mbar_init(&b_empty[i], 1); }
        for (int i = 0; i < 2; i++) { mbar_init(&t_full[i], 1); mbar_init(&t_empty[i], 128); }
        fence_barrier_init();
    }
    if (warp == 2) tmem_alloc(tmem_slot, tmem_cols);
    for (int i = threadIdx.x; i < p.N; i += blockDim.x) {
        s_bias[i] = p.bias[i];
        if (p.out_kind == 3) s_w2[i] = p.w2[i];
    }
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem_base = *tmem_slot;

    if (warp == 0) {
        // ===== producer: halo (A) and weight (B) bulk copies =====
        if (lane == 0) {
            uint32_t as = 0, ap = 0, bs = 0, bp = 0;
            for (int tile = blockIdx.x; tile < p.ntiles; tile += gridDim.x) {
                const int64_t q0 = (int64_t)tile * kTileM * MT;
                int tap_pos = 0;
                for (int cb = 0; cb < p.ncb; cb++) {
                    tap_pos = 0;
                    for (int g = 0; g < p.ngroups; g++) {
                        mbar_wait(&a_empty[as], ap ^ 1);
                        mbar_arrive_expect_tx(&a_full[as], a_bytes);
                        uint8_t *dst = a_buf + (size_t)as * a_bytes;
                        const int plane = p.group_plane[g];
                        for (uint32_t j = 0; j < chunks; j++) {
                            const uint8_t *src =
                                p.act + (((int64_t)plane * p.c8_in + cb * chunks + j) * p.lcap + q0) * 16;
                            bulk_g2s(dst + j * p.P * 16, src, p.P * 16, &a_full[as]);
                        }
                        if (++as == (uint32_t)p.stages_a) { as = 0; ap ^= 1; }
                        for (int t = 0; t < p.group_ntaps[g]; t++, tap_pos++) {
                            mbar_wait(&b_empty[bs], bp ^ 1);
                            mbar_arrive_expect_tx(&b_full[bs], b_bytes);
                            bulk_g2s(b_buf + (size_t)bs * b_bytes, p.wpk + ((size_t)cb * 9 + tap_pos) * b_bytes, b_bytes,
                                     &b_full[bs]);
                            if (++bs == (uint32_t)p.stages_b) { bs = 0; bp ^= 1; }
                        }
                    }
                }
            }
        }
    } else if (warp == 1) {
        // ===== MMA issuer (single thread) =====
        if (lane == 0) {
            const uint32_t idesc = SWAP ? umma_idesc_bf16(kTileM, kTileM * MT) : umma_idesc_bf16(kTileM, p.N);
            uint32_t as = 0, ap = 0, bs = 0, bp = 0, acc = 0, accp = 0;
            const uint32_t a_base = smem_u32(a_buf), b_base = smem_u32(b_buf);
            const uint32_t lbo_a = p.P * 16, lbo_b = p.N * 16;
            for (int tile = blockIdx.x; tile < p.ntiles; tile += gridDim.x) {
                mbar_wait(&t_empty[acc], accp ^ 1);
                tc_fence_after();
                const uint32_t d = tmem_base + acc * MT * p.N;
                uint32_t accumulate = 0;
                for (int cb = 0; cb < p.ncb; cb++) {
                    for (int g = 0; g < p.ngroups; g++) {
                        mbar_wait(&a_full[as], ap);
                        tc_fence_after();
                        const uint32_t a_stage = a_base + as * a_bytes;
                        for (int t = 0; t < p.group_ntaps[g]; t++) {
                            mbar_wait(&b_full[bs], bp);
                            tc_fence_after();
                            const uint32_t a_tap = a_stage + p.group_shift[g][t] * 16;
                            const uint32_t b_stage = b_base + bs * b_bytes;
                            for (uint32_t s = 0; s < chunks / 2; s++) {
                                const uint64_t bd = umma_desc(b_stage + 2 * s * lbo_b, lbo_b, 128);
                                if (SWAP) {
                                    // weights = M operand, the 128*MT halo rows = N operand
                                    const uint64_t hd = umma_desc(a_tap + 2 * s * lbo_a, lbo_a, 128);
                                    umma_bf16(d, bd, hd, idesc, accumulate);
                                } else {
                                    // the mt sub-tiles share this B stage: rows 128*m.. of the halo
#pragma unroll
                                    for (int m = 0; m < MT; m++) {
                                        uint64_t ad = umma_desc(a_tap + 2 * s * lbo_a + m * (kTileM * 16), lbo_a, 128);
                                        umma_bf16(d + m * p.N, ad, bd, idesc, accumulate);
                                    }
                                }
                                accumulate = 1;
                            }
                            umma_commit(&b_empty[bs]);
                            if (++bs == (uint32_t)p.stages_b) { bs = 0; bp ^= 1; }
                        }
                        umma_commit(&a_empty[as]);
                        if (++as == (uint32_t)p.stages_a) { as = 0; ap ^= 1; }
                    }
                }
                umma_commit(&t_full[acc]);
                if (++acc == 2) { acc = 0; accp ^= 1; }
            }
        }
    } else if (SWAP && warp >= 4) {
        // ===== head epilogue, transposed accumulator: lane = D1 channel, column = pixel =====
        const int quarter = warp & 3;
        const int ch = quarter * 32 + lane;
        const float bias_c = s_bias[ch], w2_c = s_w2[ch];
        const int r = threadIdx.x - 128;
        uint32_t acc = 0, accp = 0;
        for (int tile = blockIdx.x; tile < p.ntiles; tile += gridDim.x) {
            mbar_wait(&t_full[acc], accp);
            tc_fence_after();
            const uint32_t taddr = tmem_base + ((uint32_t)(quarter * 32) << 16) + acc * (kTileM * MT);
            for (int cc = 0; cc < kTileM * MT / 32; cc++) {
                uint32_t v[32];
                tmem_ld32(taddr + cc * 32, v);
                float t[32];
#pragma unroll
                for (int j = 0; j < 32; j += 2) {
                    const uint32_t pk = pack_bf16x2(fmaxf(__uint_as_float(v[j]) + bias_c, 0.0f),
                                                    fmaxf(__uint_as_float(v[j + 1]) + bias_c, 0.0f));
                    t[j] = w2_c * __uint_as_float(pk << 16);
                    t[j + 1] = w2_c * __uint_as_float(pk & 0xFFFF0000u);
                }
                // reduce-scatter over the 32 channels of this warp: lane l ends with pixel l
#pragma unroll
                for (int sft = 16; sft >= 1; sft >>= 1) {
                    const bool up = (lane & sft) != 0;
#pragma unroll
                    for (int j = 0; j < sft; j++) {
                        const float send = up ? t[j] : t[j + sft];
                        const float keep = up ? t[j + sft] : t[j];
                        t[j] = keep + __shfl_xor_sync(0xffffffffu, send, sft);
                    }
                }
                s_red[quarter * (kTileM * MT) + cc * 32 + lane] = t[0];
            }
            tc_fence_before();
            mbar_arrive(&t_empty[acc]);
            asm volatile("bar.sync 1, 128;" ::: "memory");
            for (int px = r; px < kTileM * MT; px += 128) {
                const float z = p.b2 + ((s_red[px] + s_red[kTileM * MT + px]) +
                                        (s_red[2 * kTileM * MT + px] + s_red[3 * kTileM * MT + px]));
                const int64_t q = (int64_t)tile * kTileM * MT + px;
                const int f = (int)(q / p.fstride);
                const int64_t rr = q - (int64_t)f * p.fstride;
                const int oy = (int)(rr / p.pitch);
                const int ox = (int)(rr - (int64_t)oy * p.pitch);
                if (q < p.mtot && oy < p.out_h && ox < p.out_w)
                    p.scores[((int64_t)f * p.out_h + oy) * p.out_w + ox] = 1.0f / (1.0f + expf(-z));
            }
            asm volatile("bar.sync 1, 128;" ::: "memory");
            if (++acc == 2) { acc = 0; accp ^= 1; }
        }
    } else if (warp >= 4) {
        // ===== epilogue: TMEM -> regs -> bias, ReLU, bf16 -> next layer's layout =====
        const int row = threadIdx.x - 128;          // TMEM lane == tile row
        const int quarter = warp & 3;               // lanes 32*quarter .. +31
        uint32_t acc = 0, accp = 0;
        for (int tile = blockIdx.x; tile < p.ntiles; tile += gridDim.x) {
            mbar_wait(&t_full[acc], accp);
            tc_fence_after();
          for (int m = 0; m < MT; m++) {
            const int64_t q = (int64_t)tile * kTileM * MT + m * kTileM + row;
            const int f = (int)(q / p.fstride);
            const int64_t r = q - (int64_t)f * p.fstride;
            const int oy = (int)(r / p.pitch);
            const int ox = (int)(r - (int64_t)oy * p.pitch);
            const bool valid = q < p.mtot && oy < p.out_h && ox < p.out_w;
            int plane = 0;
            int64_t L = 0;
            if (p.out_kind != 3) L = layout_pixel(p.out_kind, p.out_pitch, p.out_fstride, f, oy, ox, plane);
            const uint32_t taddr = tmem_base + ((uint32_t)(quarter * 32) << 16) + (acc * MT + m) * p.N;
            float z = p.b2;
            for (int cc = 0; cc < p.N / 32; cc++) {
                uint32_t v[32];
                tmem_ld32(taddr + cc * 32, v);
                uint32_t pk[16];
#pragma unroll
                for (int j = 0; j < 16; j++) {
                    float a = fmaxf(__uint_as_float(v[2 * j]) + s_bias[cc * 32 + 2 * j], 0.0f);
                    float b = fmaxf(__uint_as_float(v[2 * j + 1]) + s_bias[cc * 32 + 2 * j + 1], 0.0f);
                    pk[j] = pack_bf16x2(a, b);
                }
                if (p.out_kind == 3) {
#pragma unroll
                    for (int j = 0; j < 16; j++) {
                        float a = __uint_as_float(pk[j] << 16);
                        float b = __uint_as_float(pk[j] & 0xFFFF0000u);
                        z = fmaf(s_w2[cc * 32 + 2 * j], a, z);
                        z = fmaf(s_w2[cc * 32 + 2 * j + 1], b, z);
                    }
                } else if (valid) {
#pragma unroll
                    for (int c = 0; c < 4; c++) {
                        uint8_t *dst = p.out + (((int64_t)plane * p.out_c8 + cc * 4 + c) * p.out_lcap + L) * 16;
                        *reinterpret_cast<uint4 *>(dst) = make_uint4(pk[4 * c], pk[4 * c + 1], pk[4 * c + 2], pk[4 * c + 3]);
                    }
                }
            }
            if (p.out_kind == 3 && valid)
                p.scores[((int64_t)f * p.out_h + oy) * p.out_w + ox] = 1.0f / (1.0f + expf(-z));
          }
            tc_fence_before();
            mbar_arrive(&t_empty[acc]);
            if (++acc == 2) { acc = 0; accp ^= 1; }
        }
    }
    __syncwarp();
    tc_fence_before();
    __syncthreads();
    if (warp == 2) {
        tc_fence_after();
        tmem_dealloc(tmem_base, tmem_cols);
    }
}

// ---------------------------------------------------------------------------
// The same implicit GEMM on a CTA PAIR (cluster of 2, tcgen05 cta_group::2): one M=256
// MMA spans both SMs — each CTA holds 128 rows of A (its own halo) and HALF of the N
// columns of B, so per-SM shared-memory operand traffic and weight streaming halve
// (N=128 layers are otherwise shared-memory-bandwidth bound).  The leader (rank 0)
// issues the MMAs and commits them to both CTAs' barriers (multicast); the peer's MMA
// warp relays "stage full" to the leader (remote mbarrier arrive); both epilogues
// drain their own TMEM and report to the leader's accumulator-empty barrier.
// Weights are packed [cb][tap][half][chunk][N/2][8].
// ---------------------------------------------------------------------------
template <int MT>
__global__ void __launch_bounds__(kConvThreads, 1) conv_umma2_kernel(const __grid_constant__ ConvParams p) {
    extern __shared__ __align__(1024) uint8_t smem[];
    const int warp = threadIdx.x >> 5;
    const int lane = threadIdx.x & 31;
    const uint32_t rank = cluster_ctarank();
    const int cluster = blockIdx.x >> 1, nclusters = gridDim.x >> 1;

    const uint32_t chunks = p.kb >> 3;
    const uint32_t a_bytes = chunks * p.P * 16;
    const uint32_t nh = (uint32_t)p.N / 2;           // B rows held by this CTA
    const uint32_t b_bytes = nh * p.kb * 2;
    uint8_t *a_buf = smem;
    uint8_t *b_buf = a_buf + (size_t)p.stages_a * a_bytes;
    uint64_t *bars = reinterpret_cast<uint64_t *>(b_buf + (size_t)p.stages_b * b_bytes);
    uint64_t *a_full = bars;
    uint64_t *a_empty = a_full + kMaxStagesA;
    uint64_t *b_full = a_empty + kMaxStagesA;
    uint64_t *b_empty = b_full + kMaxStagesB;
    uint64_t *a_peer = b_empty + kMaxStagesB;        // leader: peer's A stage landed
    uint64_t *b_peer = a_peer + kMaxStagesA;         // leader: peer's B stage landed
    uint64_t *t_full = b_peer + kMaxStagesB;
    uint64_t *t_empty = t_full + 2;
    uint32_t *tmem_slot = reinterpret_cast<uint32_t *>(t_empty + 2);
    float *s_bias = reinterpret_cast<float *>(tmem_slot + 4);
    float *s_w2 = s_bias + 256;

    const uint32_t acc_cols = 2 * MT * p.N;
    const uint32_t tmem_cols = acc_cols <= 32 ? 32 : (acc_cols <= 64 ? 64 : (acc_cols <= 128 ? 128 : (acc_cols <= 256 ? 256 : 512)));
    const int npairs = p.ntiles;                     // pair tiles of 2 x 128*MT rows

    if (threadIdx.x == 0) {
        for (int i = 0; i < p.stages_a; i++) { mbar_init(&a_full[i], 1); mbar_init(&a_empty[i], 1); mbar_init(&a_peer[i], 1); }
        for (int i = 0; i < p.stages_b; i++) { mbar_init(&b_full[i], 1); mbar_init(&b_empty[i], 1); mbar_init(&b_peer[i], 1); }
        for (int i = 0; i < 2; i++) { mbar_init(&t_full[i], 1); mbar_init(&t_empty[i], 129);  /* 128 local + 1 from the peer */ }
        fence_barrier_init();
    }
    if (warp == 2) tmem_alloc2(tmem_slot, tmem_cols);
    for (int i = threadIdx.x; i < p.N; i += blockDim.x) {
        s_bias[i] = p.bias[i];
        if (p.out_kind == 3) s_w2[i] = p.w2[i];
    }
    tc_fence_before();
    __syncthreads();
    cluster_sync();  // both CTAs' barriers initialised before any remote arrive
    tc_fence_after();
    const uint32_t tmem_base = *tmem_slot;

    if (warp == 0) {
        // ===== producer (both CTAs): own halo rows and own half of the weights =====
        if (lane == 0) {
            uint32_t as = 0, ap = 0, bs = 0, bp = 0;
            for (int pt = cluster; pt < npairs; pt += nclusters) {
                const int64_t q0 = ((int64_t)pt * 2 + rank) * kTileM * MT;
                for (int cb = 0; cb < p.ncb; cb++) {
                    int tap_pos = 0;
                    for (int g = 0; g < p.ngroups; g++) {
                        mbar_wait(&a_empty[as], ap ^ 1);
                        mbar_arrive_expect_tx(&a_full[as], a_bytes);
                        uint8_t *dst = a_buf + (size_t)as * a_bytes;
                        const int plane = p.group_plane[g];
                        for (uint32_t j = 0; j < chunks; j++) {
                            const uint8_t *src =
                                p.act + (((int64_t)plane * p.c8_in + cb * chunks + j) * p.lcap + q0) * 16;
                            bulk_g2s(dst + j * p.P * 16, src, p.P * 16, &a_full[as]);
                        }
                        if (++as == (uint32_t)p.stages_a) { as = 0; ap ^= 1; }
                        for (int t = 0; t < p.group_ntaps[g]; t++, tap_pos++) {
                            mbar_wait(&b_empty[bs], bp ^ 1);
                            mbar_arrive_expect_tx(&b_full[bs], b_bytes);
                            bulk_g2s(b_buf + (size_t)bs * b_bytes,
                                     p.wpk + (((size_t)cb * 9 + tap_pos) * 2 + rank) * b_bytes, b_bytes, &b_full[bs]);
                            if (++bs == (uint32_t)p.stages_b) { bs = 0; bp ^= 1; }
                        }
                    }
                }
            }
        }
    } else if (warp == 1 && rank == 1) {
        // ===== peer: relay "stage full" to the leader's a_peer / b_peer =====
        if (lane == 0) {
            uint32_t as = 0, ap = 0, bs = 0, bp = 0;
            const uint32_t a_peer0 = mapa_shared(smem_u32(a_peer), 0), b_peer0 = mapa_shared(smem_u32(b_peer), 0);
            for (int pt = cluster; pt < npairs; pt += nclusters) {
                for (int cb = 0; cb < p.ncb; cb++) {
                    for (int g = 0; g < p.ngroups; g++) {
                        mbar_wait(&a_full[as], ap);
                        mbar_arrive_cluster(a_peer0 + as * 8);
                        if (++as == (uint32_t)p.stages_a) { as = 0; ap ^= 1; }
                        for (int t = 0; t < p.group_ntaps[g]; t++) {
                            mbar_wait(&b_full[bs], bp);
                            mbar_arrive_cluster(b_peer0 + bs * 8);
                            if (++bs == (uint32_t)p.stages_b) { bs = 0; bp ^= 1; }
                        }
                    }
                }
            }
        }
    } else if (warp == 1) {
        // ===== leader: MMA issuer for the pair (single thread) =====
        if (lane == 0) {
            const uint32_t idesc = umma_idesc_bf16(2 * kTileM, p.N);
            uint32_t as = 0, ap = 0, bs = 0, bp = 0, acc = 0, accp = 0;
            const uint32_t a_base = smem_u32(a_buf), b_base = smem_u32(b_buf);
            const uint32_t lbo_a = p.P * 16, lbo_b = nh * 16;
            for (int pt = cluster; pt < npairs; pt += nclusters) {
                mbar_wait_cluster(&t_empty[acc], accp ^ 1);
                tc_fence_after();
                const uint32_t d = tmem_base + acc * MT * p.N;
                uint32_t accumulate = 0;
                for (int cb = 0; cb < p.ncb; cb++) {
                    for (int g = 0; g < p.ngroups; g++) {
                        mbar_wait(&a_full[as], ap);
                        mbar_wait_cluster(&a_peer[as], ap);
                        tc_fence_after();
                        const uint32_t a_stage = a_base + as * a_bytes;
                        for (int t = 0; t < p.group_ntaps[g]; t++) {
                            mbar_wait(&b_full[bs], bp);
                            mbar_wait_cluster(&b_peer[bs], bp);
                            tc_fence_after();
                            const uint32_t a_tap = a_stage + p.group_shift[g][t] * 16;
                            const uint32_t b_stage = b_base + bs * b_bytes;
                            for (uint32_t s = 0; s < chunks / 2; s++) {
                                const uint64_t bd = umma_desc(b_stage + 2 * s * lbo_b, lbo_b, 128);
#pragma unroll
                                for (int m = 0; m < MT; m++) {
                                    uint64_t ad = umma_desc(a_tap + 2 * s * lbo_a + m * (kTileM * 16), lbo_a, 128);
                                    umma2_bf16(d + m * p.N, ad, bd, idesc, accumulate);
                                }
                                accumulate = 1;
                            }
                            umma2_commit_mc(&b_empty[bs], 0x3);
                            if (++bs == (uint32_t)p.stages_b) { bs = 0; bp ^= 1; }
                        }
                        umma2_commit_mc(&a_empty[as], 0x3);
                        if (++as == (uint32_t)p.stages_a) { as = 0; ap ^= 1; }
                    }
                }
                umma2_commit_mc(&t_full[acc], 0x3);
                if (++acc == 2) { acc = 0; accp ^= 1; }
            }
        }
    } else if (warp >= 4) {
        // ===== epilogue (both CTAs): own 128 TMEM lanes = own rows =====
        const int row = threadIdx.x - 128;
        const int quarter = warp & 3;
        const uint32_t t_empty0 = mapa_shared(smem_u32(t_empty), 0);
        uint32_t acc = 0, accp = 0;
        for (int pt = cluster; pt < npairs; pt += nclusters) {
            mbar_wait(&t_full[acc], accp);
            tc_fence_after();
            for (int m = 0; m < MT; m++) {
                const int64_t q = ((int64_t)pt * 2 + rank) * kTileM * MT + m * kTileM + row;
                const int f = (int)(q / p.fstride);
                const int64_t r = q - (int64_t)f * p.fstride;
                const int oy = (int)(r / p.pitch);
                const int ox = (int)(r - (int64_t)oy * p.pitch);
                const bool valid = q < p.mtot && oy < p.out_h && ox < p.out_w;
                int plane = 0;
                int64_t L = 0;
                if (p.out_kind != 3) L = layout_pixel(p.out_kind, p.out_pitch, p.out_fstride, f, oy, ox, plane);
                const uint32_t taddr = tmem_base + ((uint32_t)(quarter * 32) << 16) + (acc * MT + m) * p.N;
                float z = p.b2;
                for (int cc = 0; cc < p.N / 32; cc++) {
                    uint32_t v[32];
                    tmem_ld32(taddr + cc * 32, v);
                    uint32_t pk[16];
#pragma unroll
                    for (int j = 0; j < 16; j++) {
                        float a = fmaxf(__uint_as_float(v[2 * j]) + s_bias[cc * 32 + 2 * j], 0.0f);
                        float b = fmaxf(__uint_as_float(v[2 * j + 1]) + s_bias[cc * 32 + 2 * j + 1], 0.0f);
                        pk[j] = pack_bf16x2(a, b);
                    }
                    if (p.out_kind == 3) {
#pragma unroll
                        for (int j = 0; j < 16; j++) {
                            float a = __uint_as_float(pk[j] << 16);
                            float b = __uint_as_float(pk[j] & 0xFFFF0000u);
                            z = fmaf(s_w2[cc * 32 + 2 * j], a, z);
                            z = fmaf(s_w2[cc * 32 + 2 * j + 1], b, z);
                        }
                    } else if (valid) {
#pragma unroll
                        for (int c = 0; c < 4; c++) {
                            uint8_t *dst = p.out + (((int64_t)plane * p.out_c8 + cc * 4 + c) * p.out_lcap + L) * 16;
                            *reinterpret_cast<uint4 *>(dst) =
                                make_uint4(pk[4 * c], pk[4 * c + 1], pk[4 * c + 2], pk[4 * c + 3]);
                        }
                    }
                }
                if (p.out_kind == 3 && valid)
                    p.scores[((int64_t)f * p.out_h + oy) * p.out_w + ox] = 1.0f / (1.0f + expf(-z));
            }
            tc_fence_before();
            if (rank == 0) {
                mbar_arrive(&t_empty[acc]);
            } else {  // one cluster-scope release for the whole peer epilogue
                asm volatile("bar.sync 1, 128;" ::: "memory");
                if (row == 0) mbar_arrive_cluster(t_empty0 + acc * 8);
            }
            if (++acc == 2) { acc = 0; accp ^= 1; }
        }
    }
    __syncwarp();
    tc_fence_before();
    __syncthreads();
    cluster_sync();  // the peer's smem / TMEM stay alive until the pair's last MMA drained
    if (warp == 2) {
        tc_fence_after();
        tmem_dealloc2(tmem_base, tmem_cols);
    }
}

// ---------------------------------------------------------------------------
// host side: plan, weight packing, launch
// ---------------------------------------------------------------------------
static uint16_t f32_to_bf16_rne(float f) {
    uint32_t u;
    memcpy(&u, &f, 4);
    uint32_t lsb = (u >> 16) & 1u;
    u += 0x7FFFu + lsb;
    return (uint16_t)(u >> 16);
}
static float bf16_to_f32(uint16_t b) {
    uint32_t u = (uint32_t)b << 16;
    float f;
    memcpy(&f, &u, 4);
    return f;
}

struct GemmLayer {
    int cin, cout, stride, in_h, in_w, out_h, out_w;
    int kind;                     // input layout kind
    int pitch;
    int64_t fstride_unit;         // per-frame pixels of the input layout
    int max_shift;
    int ngroups, group_plane[4], group_ntaps[4], group_shift[4][9], group_tap[4][9];
    int kb, ncb, P, mt, cg;   // cg: 1 = single CTA, 2 = CTA pair (cta_group::2)
    uint8_t *wpk_dev;
    float *bias_dev;
};

}  // namespace otif

struct otif_proxy {
    otif_proxy_desc d;
    int gh, gw;
    int e1_oh, e1_ow;
    otif::GemmLayer L[5];         // E2, E3, E4, E5, D1
    uint16_t *e1_w_dev;           // [4][32][8] bf16 (K = 27 padded to 32)
    float *e1_b_dev;              // [32]
    float *w2_dev;                // [dec] bf16-rounded
    float b2;
    int num_sms;
    int head_swap;                // swapped-operand head layer (default on; OTIF_HEAD_SWAP=0 for A/B runs)
    uint64_t plan_hash;
};

namespace otif {

static void build_layer(GemmLayer &g, int cin, int cout, int stride, int in_h, int in_w) {
    g.cin = cin; g.cout = cout; g.stride = stride; g.in_h = in_h; g.in_w = in_w;
    g.out_h = (in_h + stride - 1) / stride;
    g.out_w = (in_w + stride - 1) / stride;
    g.kb = cin < 64 ? cin : 64;
    g.ncb = cin / g.kb;
    for (int i = 0; i < 4; i++) g.group_ntaps[i] = 0;
    if (stride == 1) {
        g.kind = 1;
        g.pitch = in_w + 2;
        g.fstride_unit = (int64_t)(in_h + 1) * g.pitch;
        g.max_shift = 2 * g.pitch + 2;
        g.ngroups = 1;
        g.group_plane[0] = 0;
        for (int t = 0; t < 9; t++) {
            g.group_tap[0][t] = t;
            g.group_shift[0][t] = (t / 3) * g.pitch + (t % 3);
        }
        g.group_ntaps[0] = 9;
    } else {
        g.kind = 2;
        g.pitch = g.out_w + 1;
        g.fstride_unit = (int64_t)(g.out_h + 1) * g.pitch;
        g.max_shift = g.pitch + 1;
        // plane (rp, cp): rp = (kh != 1), cp = (kw != 1); shift = (kh != 0)*pitch + (kw != 0)
        int ng = 0;
        for (int plane = 0; plane < 4; plane++) {
            int cnt = 0;
            for (int t = 0; t < 9; t++) {
                int kh = t / 3, kw = t % 3;
                int pl = ((kh != 1) << 1) | (kw != 1);
                if (pl != plane) continue;
                g.group_tap[ng][cnt] = t;
                g.group_shift[ng][cnt] = (kh != 0) * g.pitch + (kw != 0);
                cnt++;
            }
            g.group_plane[ng] = plane;
            g.group_ntaps[ng] = cnt;
            ng++;
        }
        g.ngroups = ng;
    }
    // mt sub-tiles of 128 rows per CTA tile so that every tap issues >= 256 columns of MMA
    // work (mt * N = 256): amortises the per-stage barrier and copy overheads of small N
    g.mt = cout >= 256 ? 1 : (cout >= 128 ? 2 : 4);
    // CTA pairs (cta_group::2) would halve per-SM operand traffic for N >= 128, but with
    // the relayed stage hand-off they measured 1.3-1.7x SLOWER than single CTAs on B200
    // (profiles/r01_cta_pair.md); single CTAs are the default, pairs opt-in for tuning.
    g.cg = 1;
    if (const char *e = getenv("OTIF_CONV_CG")) {  // tuning experiments only
        if (atoi(e) == 2 && cout >= 128) g.cg = 2;
    }
    if (const char *e = getenv("OTIF_CONV_MT_MAX")) {  // tuning experiments only
        int cap = atoi(e);
        if (cap >= 1 && g.mt > cap) g.mt = cap;
    }
    g.P = (int)round_up(kTileM * g.mt + g.max_shift, 8);
}

static Layout input_layout(const GemmLayer &g, int n) {
    Layout l;
    l.kind = g.kind;
    l.planes = g.kind == 1 ? 1 : 4;
    l.pitch = g.pitch;
    l.fstride = g.fstride_unit;
    int64_t mtot = (int64_t)n * g.fstride_unit;
    l.lcap = round_up(round_up(mtot, (int64_t)kTileM * g.mt * g.cg) + g.max_shift + 8, 16);
    l.c8 = g.cin / 8;
    l.bytes = (size_t)l.planes * l.c8 * l.lcap * 16;
    l.offset = 0;
    return l;
}

static size_t plan_workspace(const otif_proxy *p, int n, Layout lay[5]) {
    size_t off = 256;  // tag header
    for (int i = 0; i < 5; i++) {
        lay[i] = input_layout(p->L[i], n);
        lay[i].offset = off;
        off += round_up(lay[i].bytes, 256);
    }
    return off;
}

static void conv_smem(const GemmLayer &g, int &sa, int &sb, size_t &bytes) {
    size_t a = (size_t)(g.kb / 8) * g.P * 16;
    size_t b = (size_t)g.cout * g.kb * 2 / g.cg;
    size_t fixed = (3 * kMaxStagesA + 3 * kMaxStagesB + 4) * 8 + 16 + 2 * 256 * 4 + 4 * 256 * 4 + 1024;
    size_t budget = 220 * 1024;
    sa = 2; sb = 2;
    // grow B (weights stream every tap) first, then A
    // a CTA pair recycles a stage over a longer loop (peer relay, multicast commit): deeper B ring
    const int sb_max = g.cg == 2 ? kMaxStagesB : 6;
    while (sb < kMaxStagesB && sa * a + (sb + 1) * b + fixed <= budget && sb < sb_max) sb++;
    while (sa < kMaxStagesA && (sa + 1) * a + sb * b + fixed <= budget && sa < 3) sa++;
    bytes = sa * a + sb * b + fixed;
}

// evs (optional): 6 events recorded after E1 (prep) and after each of the 5 GEMM layers
otif_status launch_proxy(const otif_proxy *p, const uint8_t *img, int n, float *scores, uint8_t *ws,
                         size_t ws_bytes, cudaStream_t stream, cudaEvent_t *evs) {
    Layout lay[5];
    size_t need = plan_workspace(p, n, lay);
    if (ws_bytes < need) {
        set_error("otif_proxy_score: workspace %zu B < required %zu B", ws_bytes, need);
        return OTIF_ENOMEM;
    }
    // Lay the buffers out for the largest batch this workspace can hold, so that every
    // batch size up to it shares one layout (and one zero-initialisation): a smaller
    // final batch then does not re-zero the workspace.
    int n_plan = n;
    {
        int64_t lo = n, hi = n;
        while (hi < (1 << 24) && plan_workspace(p, (int)(hi * 2), lay) <= ws_bytes) hi *= 2;
        int64_t top = hi * 2;
        lo = hi;
        while (top - lo > 1) {  // largest m in [hi, 2hi) with bytes(m) <= ws_bytes
            int64_t mid = (lo + top) / 2;
            if (plan_workspace(p, (int)mid, lay) <= ws_bytes) lo = mid;
            else top = mid;
        }
        n_plan = (int)lo;
        need = plan_workspace(p, n_plan, lay);
    }
    const uint64_t tag = p->plan_hash ^ ((uint64_t)n_plan * 0x9E3779B97F4A7C15ull) ^ (uint64_t)need;
    ws_zero_kernel<<<p->num_sms * 4, 256, 0, stream>>>(ws, need, tag);
    OTIF_LAUNCH_CHECK();
    ws_tag_kernel<<<1, 1, 0, stream>>>(ws, tag);
    OTIF_LAUNCH_CHECK();

    // E1
    {
        E1Params e;
        e.img = img; e.n = n; e.h = p->d.in_h; e.w = p->d.in_w; e.oh = p->e1_oh; e.ow = p->e1_ow;
        e.bias = p->e1_b_dev;
        e.out_kind = lay[0].kind; e.out_pitch = lay[0].pitch; e.out_fstride = lay[0].fstride;
        e.out_lcap = lay[0].lcap; e.out = ws + lay[0].offset;
        e.wpk = p->e1_w_dev;
        e.ntiles = cdiv((int64_t)n * e.oh * e.ow, 128);
        int64_t blocks = e.ntiles < (int64_t)p->num_sms * 8 ? e.ntiles : (int64_t)p->num_sms * 8;
        if (blocks < 1) blocks = 1;
        e1_umma_kernel<<<(unsigned)blocks, 128, 0, stream>>>(e);
        OTIF_LAUNCH_CHECK();
        if (evs) OTIF_CUDA(cudaEventRecord(evs[0], stream));
    }
    // E2..E5, D1
    for (int li = 0; li < 5; li++) {
        const GemmLayer &g = p->L[li];
        ConvParams c;
        memset(&c, 0, sizeof(c));
        c.act = ws + lay[li].offset;
        c.lcap = lay[li].lcap;
        c.c8_in = g.cin / 8;
        c.kb = g.kb; c.ncb = g.ncb; c.P = g.P; c.ngroups = g.ngroups; c.mt = g.mt;
        for (int i = 0; i < 4; i++) {
            c.group_plane[i] = g.group_plane[i];
            c.group_ntaps[i] = g.group_ntaps[i];
            for (int t = 0; t < 9; t++) c.group_shift[i][t] = g.group_shift[i][t];
        }
        c.wpk = g.wpk_dev; c.bias = g.bias_dev; c.N = g.cout;
        c.mtot = (int64_t)n * g.fstride_unit;
        c.ntiles = (int)cdiv(c.mtot, (int64_t)kTileM * g.mt * g.cg);  // pair tiles when cg == 2
        c.pitch = g.pitch; c.fstride = g.fstride_unit; c.out_h = g.out_h; c.out_w = g.out_w;
        if (li < 4) {
            c.out_kind = lay[li + 1].kind;
            c.out = ws + lay[li + 1].offset;
            c.out_lcap = lay[li + 1].lcap;
            c.out_c8 = lay[li + 1].c8;
            c.out_pitch = lay[li + 1].pitch;
            c.out_fstride = lay[li + 1].fstride;
        } else {
            c.out_kind = 3;
            c.scores = scores;
            c.w2 = p->w2_dev;
            c.b2 = p->b2;
        }
        size_t smem;
        conv_smem(g, c.stages_a, c.stages_b, smem);
        if (g.cg == 2) {
            const int pairs = p->num_sms / 2;
            const int clusters = c.ntiles < pairs ? (c.ntiles < 1 ? 1 : c.ntiles) : pairs;
            auto kern = g.mt == 4 ? conv_umma2_kernel<4> : (g.mt == 2 ? conv_umma2_kernel<2> : conv_umma2_kernel<1>);
            OTIF_CUDA(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
            cudaLaunchConfig_t cfg = {};
            cfg.gridDim = dim3(2 * clusters);
            cfg.blockDim = dim3(kConvThreads);
            cfg.dynamicSmemBytes = smem;
            cfg.stream = stream;
            cudaLaunchAttribute attr[1];
            attr[0].id = cudaLaunchAttributeClusterDimension;
            attr[0].val.clusterDim.x = 2;
            attr[0].val.clusterDim.y = 1;
            attr[0].val.clusterDim.z = 1;
            cfg.attrs = attr;
            cfg.numAttrs = 1;
            OTIF_CUDA(cudaLaunchKernelEx(&cfg, kern, c));
        } else {
            int grid = c.ntiles < p->num_sms ? c.ntiles : p->num_sms;
            if (grid < 1) grid = 1;
            // head layer with N = 128: swapped operands (see conv_umma_kernel)
            const bool swap = c.out_kind == 3 && g.mt == 2 && g.cout == 128 && p->head_swap;
            auto kern = swap ? conv_umma_kernel<2, true>
                             : (g.mt == 4 ? conv_umma_kernel<4> : (g.mt == 2 ? conv_umma_kernel<2> : conv_umma_kernel<1>));
            OTIF_CUDA(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
            kern<<<grid, kConvThreads, smem, stream>>>(c);
        }
        OTIF_LAUNCH_CHECK();
        if (evs) OTIF_CUDA(cudaEventRecord(evs[1 + li], stream));
    }
    return OTIF_OK;
}

}  // namespace otif

// ---------------------------------------------------------------------------
// C ABI
// ---------------------------------------------------------------------------
using namespace otif;

static bool width_ok(int c) { return c == 64 || c == 128 || c == 256; }

extern "C" otif_status otif_proxy_create(const otif_proxy_desc *d, const float *weights, size_t n_weights,
                                         otif_proxy **out) {
    OTIF_REQUIRE(d && weights && out, "otif_proxy_create: NULL argument");
    OTIF_REQUIRE(d->in_h > 0 && d->in_w > 0, "otif_proxy_create: bad input size %dx%d", d->in_w, d->in_h);
    OTIF_REQUIRE(d->n_strided >= 1 && d->n_strided <= 5, "otif_proxy_create: n_strided %d not in [1,5]", d->n_strided);
    if (d->enc[0] != 32 || !width_ok(d->enc[1]) || !width_ok(d->enc[2]) || !width_ok(d->enc[3]) ||
        !width_ok(d->enc[4]) || !width_ok(d->dec)) {
        set_error("otif_proxy_create: widths (%d,%d,%d,%d,%d|%d) unsupported (enc[0]=32, others in {64,128,256})",
                  d->enc[0], d->enc[1], d->enc[2], d->enc[3], d->enc[4], d->dec);
        return OTIF_EUNSUPPORTED;
    }
    int num_sms = 0;
    otif_status st = check_device(&num_sms);
    if (st != OTIF_OK) return st;

    // expected blob size
    int cin[7], cout[7], ks[7];
    {
        int c = 3;
        for (int i = 0; i < 5; i++) { cin[i] = c; cout[i] = d->enc[i]; ks[i] = 3; c = d->enc[i]; }
        cin[5] = c; cout[5] = d->dec; ks[5] = 3;
        cin[6] = d->dec; cout[6] = 1; ks[6] = 1;
    }
    size_t offs[7], total = 0;
    for (int i = 0; i < 7; i++) { offs[i] = total; total += (size_t)cout[i] * ks[i] * ks[i] * cin[i] + cout[i]; }
    OTIF_REQUIRE(n_weights == total, "otif_proxy_create: n_weights %zu != %zu for this shape", n_weights, total);

    otif_proxy *p = new (std::nothrow) otif_proxy();
    if (!p) return OTIF_ENOMEM;
    p->d = *d;
    p->num_sms = num_sms;
    {
        const char *e = getenv("OTIF_HEAD_SWAP");
        p->head_swap = !(e && e[0] == '0');
    }
    // spatial chain
    int h = d->in_h, w = d->in_w;
    int hs[7], wss[7];
    for (int i = 0; i < 6; i++) {
        hs[i] = h; wss[i] = w;
        int s = (i < 5 && i < d->n_strided) ? 2 : 1;
        h = (h + s - 1) / s; w = (w + s - 1) / s;
    }
    p->gh = h; p->gw = w;
    p->e1_oh = (d->in_h + 1) / 2;
    p->e1_ow = (d->in_w + 1) / 2;

    otif_status rc = OTIF_OK;
    std::vector<float> host;
    // E1 weights -> bf16 [chunk j][n][8], k = j*8 + e = (kh*3+kw)*3 + c, zero for k >= 27
    {
        std::vector<uint16_t> w1(4 * 32 * 8, 0);
        std::vector<float> b1(32);
        for (int o = 0; o < 32; o++) {
            for (int k = 0; k < 27; k++) {
                int kh = k / 9, kw = (k / 3) % 3, c = k % 3;
                float v = weights[offs[0] + ((size_t)(o * 3 + kh) * 3 + kw) * 3 + c];
                w1[((k / 8) * 32 + o) * 8 + (k % 8)] = f32_to_bf16_rne(v);
            }
            b1[o] = weights[offs[0] + (size_t)32 * 27 + o];
        }
        if (cudaMalloc(&p->e1_w_dev, w1.size() * 2) != cudaSuccess || cudaMalloc(&p->e1_b_dev, 32 * 4) != cudaSuccess) {
            rc = OTIF_ENOMEM;
        } else {
            cudaMemcpy(p->e1_w_dev, w1.data(), w1.size() * 2, cudaMemcpyHostToDevice);
            cudaMemcpy(p->e1_b_dev, b1.data(), 32 * 4, cudaMemcpyHostToDevice);
        }
    }
    // GEMM layers E2..E5 (layer index 1..4) and D1 (5)
    for (int li = 0; li < 5 && rc == OTIF_OK; li++) {
        int layer = li + 1;
        int s = (layer < 5 && layer < d->n_strided) ? 2 : 1;
        GemmLayer &g = p->L[li];
        build_layer(g, cin[layer], cout[layer], s, hs[layer], wss[layer]);
        // pack: [cb][tap in loop order][chunk j][n][8]
        const int chunks = g.kb / 8;
        std::vector<uint16_t> pk((size_t)g.ncb * 9 * chunks * g.cout * 8);
        const float *W = weights + offs[layer];
        for (int cb = 0; cb < g.ncb; cb++) {
            int pos = 0;
            for (int gi = 0; gi < g.ngroups; gi++)
                for (int t = 0; t < g.group_ntaps[gi]; t++, pos++) {
                    int tap = g.group_tap[gi][t];
                    int kh = tap / 3, kw = tap % 3;
                    for (int j = 0; j < chunks; j++)
                        for (int nn = 0; nn < g.cout; nn++)
                            for (int e = 0; e < 8; e++) {
                                int ci = cb * g.kb + j * 8 + e;
                                float v = W[(((size_t)nn * 3 + kh) * 3 + kw) * g.cin + ci];
                                // cg == 2: [cb][tap][half][chunk][N/2][8] (each CTA of a pair streams its half)
                                const int nh = g.cout / g.cg, half = nn / nh, nl = nn - half * nh;
                                pk[(((((size_t)cb * 9 + pos) * g.cg + half) * chunks + j) * nh + nl) * 8 + e] =
                                    f32_to_bf16_rne(v);
                            }
                }
        }
        std::vector<float> bias(g.cout);
        for (int nn = 0; nn < g.cout; nn++) bias[nn] = W[(size_t)g.cout * 9 * g.cin + nn];
        if (cudaMalloc(&g.wpk_dev, pk.size() * 2) != cudaSuccess || cudaMalloc(&g.bias_dev, g.cout * 4) != cudaSuccess) {
            rc = OTIF_ENOMEM;
            break;
        }
        cudaMemcpy(g.wpk_dev, pk.data(), pk.size() * 2, cudaMemcpyHostToDevice);
        cudaMemcpy(g.bias_dev, bias.data(), g.cout * 4, cudaMemcpyHostToDevice);
    }
    // D2 head
    if (rc == OTIF_OK) {
        std::vector<float> w2(d->dec);
        for (int c = 0; c < d->dec; c++) w2[c] = bf16_to_f32(f32_to_bf16_rne(weights[offs[6] + c]));
        p->b2 = weights[offs[6] + d->dec];
        if (cudaMalloc(&p->w2_dev, d->dec * 4) != cudaSuccess) rc = OTIF_ENOMEM;
        else cudaMemcpy(p->w2_dev, w2.data(), d->dec * 4, cudaMemcpyHostToDevice);
    }
    // smem feasibility
    for (int li = 0; li < 5 && rc == OTIF_OK; li++) {
        int sa, sb;
        size_t bytes;
        conv_smem(p->L[li], sa, sb, bytes);
        if (bytes > 227 * 1024) {
            set_error("otif_proxy_create: layer %d needs %zu B of shared memory (input too wide)", li + 2, bytes);
            rc = OTIF_EUNSUPPORTED;
        }
    }
    if (cudaGetLastError() != cudaSuccess && rc == OTIF_OK) rc = OTIF_ECUDA;
    if (rc != OTIF_OK) {
        otif_proxy_destroy(p);
        return rc;
    }
    uint64_t hsh = 1469598103934665603ull;
    auto mix = [&](uint64_t v) { hsh = (hsh ^ v) * 1099511628211ull; };
    mix(d->in_h); mix(d->in_w); mix(d->n_strided);
    for (int i = 0; i < 5; i++) mix(d->enc[i]);
    mix(d->dec);
    p->plan_hash = hsh | 1;
    *out = p;
    return OTIF_OK;
}

extern "C" void otif_proxy_destroy(otif_proxy *p) {
    if (!p) return;
    for (int i = 0; i < 5; i++) {
        if (p->L[i].wpk_dev) cudaFree(p->L[i].wpk_dev);
        if (p->L[i].bias_dev) cudaFree(p->L[i].bias_dev);
    }
    if (p->e1_w_dev) cudaFree(p->e1_w_dev);
    if (p->e1_b_dev) cudaFree(p->e1_b_dev);
    if (p->w2_dev) cudaFree(p->w2_dev);
    delete p;
}

extern "C" otif_status otif_proxy_grid(const otif_proxy *p, int32_t *gh, int32_t *gw) {
    OTIF_REQUIRE(p && gh && gw, "otif_proxy_grid: NULL argument");
    *gh = p->gh;
    *gw = p->gw;
    return OTIF_OK;
}

extern "C" size_t otif_proxy_workspace_bytes(const otif_proxy *p, int32_t n) {
    if (!p || n < 0) return 0;
    Layout lay[5];
    return plan_workspace(p, n, lay);
}

extern "C" otif_status otif_proxy_score(const otif_proxy *p, const uint8_t *img, int32_t n, float *scores,
                                        void *workspace, size_t ws_bytes, cudaStream_t stream) {
    OTIF_REQUIRE(p, "otif_proxy_score: NULL proxy");
    OTIF_REQUIRE(n >= 0, "otif_proxy_score: n < 0");
    if (n == 0) return OTIF_OK;
    OTIF_REQUIRE(img && scores && workspace, "otif_proxy_score: NULL pointer");
    OTIF_REQUIRE((((uintptr_t)workspace) & 255) == 0, "otif_proxy_score: workspace must be 256-B aligned");
    otif_status st = check_device(nullptr);
    if (st != OTIF_OK) return st;
    return launch_proxy(p, img, n, scores, (uint8_t *)workspace, ws_bytes, stream, nullptr);
}
