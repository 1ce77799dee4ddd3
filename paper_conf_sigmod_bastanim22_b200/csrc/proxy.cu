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
// an H x W map reads, for output pixel q, the input pixels q + kh*(W+1) + kw of the
// zero-padded map flattened row-major with pitch W+1 — a pure linear shift per tap.
// ONE pad column per row suffices: data sits in columns 1..W, and the right neighbour
// of column W is column 0 (the pad) of the next row.  So every GEMM layer's input is
// stored zero-padded and flattened, frames stacked (each frame owns H+1 rows of pitch
// W+1; the bottom pad of frame f is the top pad of frame f+1), and channel-chunk
// planar: [plane][C/8][pixels][8 bf16].  Then the
// A operand of one M tile (128 consecutive output positions) for ALL 9 taps is one
// contiguous halo of 128 + 2(W+1) + 2 pixels per 8-channel chunk, loaded once with
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

#include <cuda_fp16.h>

#include "common.cuh"
#include "packjob.cuh"

namespace otif {

// warp0 producer, warp1 MMA, warp2 TMEM alloc, warps4-7 epilogue, warps 8.. fused pack copy
#ifndef OTIF_PJ_WARPS
#define OTIF_PJ_WARPS 8          // fused copy warps per conv CTA (A/B builds)
#endif
#ifndef OTIF_PJ_UNROLL
#define OTIF_PJ_UNROLL 8         // 16-B pieces in flight per copy lane
#endif
#ifndef OTIF_PJ_LAYERS
#define OTIF_PJ_LAYERS 0x18      // GEMM layers (bit li: 0 = E2 .. 4 = D1) whose CTAs copy: E5, D1
#endif
// (measured, scripts/pj_ab.sh, profiles/r02_pack_overlap.md: hosting the copy in E4 or in
// the latency-bound E1+E2 kernel costs about as much conv time as it saves)
constexpr int kConvThreads = 256 + 32 * OTIF_PJ_WARPS;
#ifndef OTIF_E12B
#define OTIF_E12B 0   // band variant of the fused E1+E2 kernel (A/B builds: 1 = band where it fits);
#endif            // parity-exact but 1.07 vs 0.88 ms per C2 step (profiles/r02l_e12_band.md)
#define OTIF_E12B_BUILD OTIF_E12B
#ifndef OTIF_CONV_CL_LAYERS
#define OTIF_CONV_CL_LAYERS 0     // GEMM layers (bit li: 0 = E2 .. 4 = D1) run as weight-sharing CTA pairs:
#endif                            // parity-exact, no faster (profiles/r02i_cta_pairs.md), so off by default
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
    // fused stage 5 of the PREVIOUS device batch (packjob.cuh): warps 8-15 drain its copy
    // units while this layer's MMAs run (the layer is tensor-bound, its HBM mostly idle)
    PackJob *pj;
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
//
// CL = 2 (cluster of two CTAs, each with its own M tiles and its own cta_group::1 MMAs):
// the weights (B stages) are shared — each CTA bulk-copies HALF of every B stage with
// .multicast::cluster into both CTAs' shared memory, and each MMA warp's "stage consumed"
// commit is multicast to both CTAs' b_empty barriers (count 2), so a stage is refilled
// only when both CTAs are done with it.  Per-SM L2 weight traffic halves (E4 / E5 stream
// 0.6-1.2 MB of weights per 128-row tile: 11-18 TB/s of L2 reads per step).  The two CTAs
// walk the same (cb, group, tap) sequence; an odd tile count gives the second CTA of the
// last pair a dummy tile (A re-read from the last tile, no stores: q >= mtot).
template <int MT, bool SWAP = false, int CL = 1>
__global__ void __launch_bounds__(kConvThreads, 1) conv_umma_kernel(const __grid_constant__ ConvParams p) {
    extern __shared__ __align__(1024) uint8_t smem[];
    const int warp = threadIdx.x >> 5;
    const int lane = threadIdx.x & 31;
    const int rank = CL == 2 ? (int)cluster_ctarank() : 0;
    const int pair0 = blockIdx.x / CL, npairs = gridDim.x / CL;
    const int ntp = (p.ntiles + CL - 1) / CL;   // tile pairs (tile = tp * CL + rank)

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
    int &s_conv_done = *reinterpret_cast<int *>(s_red + 4 * 256);   // set when the epilogue drained its last tile

    if (threadIdx.x == 0) {
        s_conv_done = 0;
        for (int i = 0; i < p.stages_a; i++) { mbar_init(&a_full[i], 1); mbar_init(&a_empty[i], 1); }
        for (int i = 0; i < p.stages_b; i++) { mbar_init(&b_full[i], 1); mbar_init(&b_empty[i], CL); }
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
    if (CL == 2) cluster_sync();   // the peer's barriers exist before any multicast reaches them
    tc_fence_after();
    const uint32_t tmem_base = *tmem_slot;

    if (warp == 0) {
        // ===== producer: halo (A) and weight (B) bulk copies =====
        if (lane == 0) {
            uint32_t as = 0, ap = 0, bs = 0, bp = 0;
            const uint32_t b_half = b_bytes / CL;
            for (int tp = pair0; tp < ntp; tp += npairs) {
                const int tile = tp * CL + rank;
                const int64_t q0 = (int64_t)(tile < p.ntiles ? tile : p.ntiles - 1) * kTileM * MT;
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
                            if (CL == 2) {   // this CTA's half of the stage, into both CTAs
                                bulk_g2s_mc(b_buf + (size_t)bs * b_bytes + rank * b_half,
                                            p.wpk + ((size_t)cb * 9 + tap_pos) * b_bytes + rank * b_half, b_half,
                                            &b_full[bs], 0x3);
                            } else {
                                bulk_g2s(b_buf + (size_t)bs * b_bytes, p.wpk + ((size_t)cb * 9 + tap_pos) * b_bytes,
                                         b_bytes, &b_full[bs]);
                            }
                            if (++bs == (uint32_t)p.stages_b) { bs = 0; bp ^= 1; }
                        }
                    }
                }
            }
        }
    } else if (warp == 1) {
        // ===== MMA issuer (whole warp, elected lane issues: descriptors stay warp-uniform) =====
        {
            const uint32_t idesc = SWAP ? umma_idesc_bf16(kTileM, kTileM * MT) : umma_idesc_bf16(kTileM, p.N);
            uint32_t as = 0, ap = 0, bs = 0, bp = 0, acc = 0, accp = 0;
            const uint32_t a_base = smem_u32(a_buf), b_base = smem_u32(b_buf);
            const uint32_t lbo_a = p.P * 16, lbo_b = p.N * 16;
            for (int tp = pair0; tp < ntp; tp += npairs) {
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
                                    umma_bf16_warp(d, bd, hd, idesc, accumulate);
                                } else {
                                    // the mt sub-tiles share this B stage: rows 128*m.. of the halo
#pragma unroll
                                    for (int m = 0; m < MT; m++) {
                                        uint64_t ad = umma_desc(a_tap + 2 * s * lbo_a + m * (kTileM * 16), lbo_a, 128);
                                        umma_bf16_warp(d + m * p.N, ad, bd, idesc, accumulate);
                                    }
                                }
                                accumulate = 1;
                            }
                            if (CL == 2) umma_commit_mc_warp(&b_empty[bs], 0x3);   // both CTAs' stage
                            else umma_commit_warp(&b_empty[bs]);
                            if (++bs == (uint32_t)p.stages_b) { bs = 0; bp ^= 1; }
                        }
                        umma_commit_warp(&a_empty[as]);
                        if (++as == (uint32_t)p.stages_a) { as = 0; ap ^= 1; }
                    }
                }
                umma_commit_warp(&t_full[acc]);
                if (++acc == 2) { acc = 0; accp ^= 1; }
            }
        }
    } else if (SWAP && warp >= 4 && warp < 8) {
        // ===== head epilogue, transposed accumulator: lane = D1 channel, column = pixel =====
        const int quarter = warp & 3;
        const int ch = quarter * 32 + lane;
        const float bias_c = s_bias[ch], w2_c = s_w2[ch];
        const int r = threadIdx.x - 128;
        uint32_t acc = 0, accp = 0;
        for (int tp = pair0; tp < ntp; tp += npairs) {
            const int tile = tp * CL + rank;   // >= ntiles: dummy tile, q >= mtot, nothing stored
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
        if (threadIdx.x == 128) *(volatile int *)&s_conv_done = 1;
    } else if (warp >= 4 && warp < 8) {
        // ===== epilogue: TMEM -> regs -> bias, ReLU, bf16 -> next layer's layout =====
        const int row = threadIdx.x - 128;          // TMEM lane == tile row
        const int quarter = warp & 3;               // lanes 32*quarter .. +31
        uint32_t acc = 0, accp = 0;
        for (int tp = pair0; tp < ntp; tp += npairs) {
            const int tile = tp * CL + rank;   // >= ntiles: dummy tile, q >= mtot, nothing stored
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
        if (threadIdx.x == 128) *(volatile int *)&s_conv_done = 1;
    } else if (warp >= 8 && p.pj) {
        // ===== fused pack of the previous batch: drain copy units until this CTA's conv
        // work is done (the rest continues in the next layer / pack_units_kernel) =====
        pj_drain_warp<OTIF_PJ_UNROLL>(p.pj, &s_conv_done, lane);
    }
    __syncwarp();
    tc_fence_before();
    __syncthreads();
    if (CL == 2) cluster_sync();   // no CTA leaves while its peer may still multicast into it
    if (warp == 2) {
        tc_fence_after();
        tmem_dealloc(tmem_base, tmem_cols);
    }
}

// ---------------------------------------------------------------------------
// E1 fused into E2 (stride-2 E2 only).  E1's output never reaches HBM: per E2 tile
// (M = 256 output positions of E2's parity-split input layout) the CTA
//   1. stages the proxy-image rows the tile needs in shared memory ("slab": 4 image
//      rows per plane row + 1; bulk copies, rows outside the frame filled with 128,
//      i.e. x = 0 after normalisation = the zero padding of P:L135's convs);
//   2. computes, one parity plane at a time ("plane job"), the E1 activations of the
//      tile's A halo (P = 128 KT rows per plane) on the tensor cores: gather warps build
//      the im2col rows from the slab as fp16 (u - 128) — exact integers — against fp16
//      weights w * 2^s (exact: bf16 has 8 significant bits), so the fp32 accumulator is
//      2^(s+7) times the bf16-path sum (power-of-two scaling commutes with rounding);
//      epilogue warps apply acc * 2^-(s+7) + b, ReLU, bf16 RNE and write the rows into a
//      plane buffer in E2's no-swizzle K-major A layout (pads exactly zero);
//   3. runs E2's taps of that plane from the plane buffer (weights resident in shared
//      memory) and drains the accumulators into E3's input layout.
// Hand-offs are per plane job (a commit + wait round trip costs ~300-470 clk on B200,
// scripts/micro/mma_rate.cu), and E1 and E2 MMAs come from two issuer warps so neither
// chain stalls the other.  Roles (768 threads): warp 0 slab loader, warp 1 E1 MMA issuer,
// warp 2 TMEM allocator, warp 3 E2 MMA issuer, warps 4-11 gather (2 warpgroups taking
// alternate E1 M tiles), 12-19 E1 epilogue (likewise), 20-23 E2 epilogue.
// Measured bound (ncu, C2): instruction fetch.  With 24 warps in 7 roles the kernel was
// "stall_no_instructions"-bound (51% of warp samples; shared-memory pipe 29%, tensor pipe
// 14%): knocking out ALL gather / epilogue / E2-tap work left 1.1 of its 1.6 ms.  The
// per-plane loops (g, taps, k sub-tiles, M sub-tiles) are therefore kept rolled
// (#pragma unroll 1): 5720 -> 3950 SASS instructions, 1.66 -> 0.97 ms per C2 step.
// TMEM: E2 accumulators 2 x 128 columns at 0, E1 accumulators 2 plane slots x 32 KT at 256.
// ---------------------------------------------------------------------------
#ifndef OTIF_PJ_E12
#define OTIF_PJ_E12 0            // fused pack copy warps in the E1+E2 kernel (A/B builds; 0 = none)
#endif
constexpr int kE12Threads = 768 + 32 * OTIF_PJ_E12;
#ifndef OTIF_E12_GATHER2
#define OTIF_E12_GATHER2 0    // 1: a thread's two im2col rows per job built together (measured neutral, r02q)
#endif
#ifndef OTIF_E12_TS
#define OTIF_E12_TS 0         // 1: E1's im2col rows in TMEM (two buffers, tcgen05.st by the gather,
#endif                        //    A-from-TMEM MMAs): 194 KB less shared-memory traffic per tile
#ifndef OTIF_E12_ACC
#define OTIF_E12_ACC (OTIF_E12_TS ? 1 : 2)   // E2 accumulator stages (A/B builds; TS needs the TMEM of one)
#endif
#ifndef OTIF_E12_E1SLOTS
#define OTIF_E12_E1SLOTS 2    // E1 accumulator slots (A/B builds; 3 needs OTIF_E12_ACC=1)
#endif
constexpr int kE12MaxPlaneBufs = 4;

struct E12Params {
    const uint8_t *img;         // u8 [n, hp, wp, 3]
    int n, hp, wp, row_bytes;   // row_bytes = 3 wp
    int h1, w1;                 // E1 output
    int h2, w2, pitch;          // E2 output; pitch = w2 + 1
    uint32_t fstride, mtot;     // E2 input layout (mtot + P < 2^31)
    FastDiv div_pitch, div_rpf, div_fstride;  // / pitch, / (h2 + 1) plane rows per frame, / fstride
    int P;                      // plane-buffer rows = 128 KT
    int np;                     // plane buffers in the ring (2 or 3)
    int na1;                    // A1 (im2col) plane stages (1 or 2)
    int ntiles;
    int slab_rows, slab_pitch;  // per slab buffer
    int bulk;                   // image rows may be bulk-copied (16-B aligned rows)
    int trace;                  // OTIF_E12_TRACE: CTA 0 prints per-role hand-off times (debug)
    int group_ntaps[4], group_shift[4][9];
    const uint16_t *wt1;        // fp16 [4 chunks][32 n][8]: K = kh*10 + kw*3 + c -> w * 2^s; K = kh*10 + 9 -> bias parts
    const uint16_t *wt2;        // bf16 [9 taps in loop order][4 chunks][64 n][8], * 2^-(s+7)
    const float *b2;
    // destination: E3's input layout
    int out_kind;
    uint8_t *out;
    int64_t out_lcap;
    int out_c8, out_pitch;
    int64_t out_fstride;
    PackJob *pj;                // fused stage 5 of the previous batch (warps 24..), or NULL
};

// Trace / knock-out bits (OTIF_E12_TRACE, read at launch) exist only in a trace build
// (nvcc -DOTIF_E12_TRACE_BUILD); in the release library they are the constant 0, so no
// environment variable can change what the shipped kernel computes.
#ifdef OTIF_E12_TRACE_BUILD
#define E12_BITS (p.trace)
#else
#define E12_BITS 0
#endif

// E2-layout position q of a tile whose first plane row is g0: which of the 4 parity
// planes hold an E1 pixel there (bit (rp << 1) | cp), and the slab byte offset of the
// image sample at (row 2y - 1, column 2x - 1) for plane (0, 0) (the other planes add
// 2 rp slab rows and 6 cp bytes).
__device__ __forceinline__ void e12_decode(const E12Params &p, uint32_t q, uint32_t g0, uint32_t &vmask,
                                           uint32_t &off) {
    const uint32_t gr = fdiv(q, p.div_pitch);
    const int j = (int)(q - gr * (uint32_t)p.pitch);
    const int i = (int)(gr - fdiv(gr, p.div_rpf) * (uint32_t)(p.h2 + 1));
    const bool in = q < p.mtot && i >= 1 && j >= 1;
    const uint32_t r1 = 2 * i - 1 < p.h1, c1 = 2 * j - 1 < p.w1;
    vmask = in ? (1u | (c1 << 1) | (r1 << 2) | ((r1 & c1) << 3)) : 0u;
    off = 4 * (gr - g0) * (uint32_t)p.slab_pitch + 12 * (uint32_t)j + 1;
}

// One im2col row of E1 (fp16, K = 32 with the bias slots) for E2-layout position with
// decode (valid, off) in parity plane (rp, cp), read from the staged image slab.
__device__ __forceinline__ void e12_im2col_row(const E12Params &p, const uint8_t *slab, uint32_t valid, uint32_t off,
                                               int rp, int cp, uint32_t (&wv)[16]) {
#pragma unroll
    for (int j = 0; j < 16; j++) wv[j] = 0;
    if (!valid || (E12_BITS & 4)) return;   // trace & 4: timing experiment (no gather)
    const uint32_t b = off + 2 * rp * p.slab_pitch + 6 * cp;
    const uint32_t sh = (b & 3) * 8;
    const uint32_t *wp = reinterpret_cast<const uint32_t *>(slab + (b & ~3u));
    uint32_t w[9];
#pragma unroll
    for (int kh = 0; kh < 3; kh++) {
        const uint32_t *r = wp + kh * (p.slab_pitch >> 2);
        w[3 * kh] = r[0]; w[3 * kh + 1] = r[1]; w[3 * kh + 2] = r[2];
    }
#pragma unroll
    for (int kh = 0; kh < 3; kh++) {
        const uint32_t w0 = w[3 * kh], w1 = w[3 * kh + 1], w2 = w[3 * kh + 2];
        const uint32_t a0 = __funnelshift_r(w0, w1, sh), a1 = __funnelshift_r(w1, w2, sh);
        wv[5 * kh + 0] = sub_f16x2(__byte_perm(a0, 0x64646464u, 0x4140), 0x64806480u);
        wv[5 * kh + 1] = sub_f16x2(__byte_perm(a0, 0x64646464u, 0x4342), 0x64806480u);
        wv[5 * kh + 2] = sub_f16x2(__byte_perm(a1, 0x64646464u, 0x4140), 0x64806480u);
        wv[5 * kh + 3] = sub_f16x2(__byte_perm(a1, 0x64646464u, 0x4342), 0x64806480u);
        // (u - 128, 128): the second half multiplies the bias part at K = 10 kh + 9
        wv[5 * kh + 4] = sub_f16x2(0x64006400u | ((w2 >> sh) & 0xFFu), 0x63006480u);
    }
}

#ifdef OTIF_E12_TRACE_BUILD   // hand-off timeline of CTA 0 (nvcc -DOTIF_E12_TRACE_BUILD; OTIF_E12_TRACE=1)
#ifndef OTIF_E12_TRACE_J0
#define OTIF_E12_TRACE_J0 0   // first traced plane job (steady state: e.g. 200)
#endif
#define E12_TR(slot, col)                                                                                 \
    do {                                                                                                  \
        if (tr && (int)J >= OTIF_E12_TRACE_J0 && (int)J < OTIF_E12_TRACE_J0 + 16)                         \
            tt[slot][J - OTIF_E12_TRACE_J0] = clock64();                                                  \
    } while (0)
#define E12_TR_DUMP(name, nslots)                                                                   \
    do {                                                                                            \
        if (tr)                                                                                     \
            for (int j_ = 0; j_ < 16; j_++)                                                         \
                printf("%s t%d J=%2d %8lld %8lld %8lld\n", name, (int)threadIdx.x, j_, tt[0][j_] - t00, (nslots) > 1 ? tt[1][j_] - t00 : 0ll, \
                       (nslots) > 2 ? tt[2][j_] - t00 : 0ll);                                       \
    } while (0)
#define E12_TR_DECL                                                       \
    const bool tr = (E12_BITS & 1) && blockIdx.x == 0 && ((threadIdx.x & 127) == 0 || threadIdx.x == 32 || threadIdx.x == 96); \
    long long tt[3][16];                                                   \
    const long long t00 = clock64();
#else
#define E12_TR(slot, col) do {} while (0)
#define E12_TR_DUMP(name, nslots) do {} while (0)
#define E12_TR_DECL
#endif

#define E12_WAIT_SLEEP(b, ph) (E12_BITS & 2 ? mbar_wait(b, ph) : mbar_wait_sleep(b, ph))
// waits on the hand-off chain (gather <- a1_empty, E1 epilogue <- a2_empty): polling (bit 128 = sleep, A/B)
#define E12_WAIT_CHAIN(b, ph) (E12_BITS & 128 ? mbar_wait_sleep(b, ph) : mbar_wait(b, ph))
template <int KT>
__global__ void __launch_bounds__(kE12Threads, 1) e12_umma_kernel(const __grid_constant__ E12Params p) {
    // TMEM: E2 accumulators kAccStages x (MT x 64) at 0, E1 accumulators kE1Slots x 32 KT
    constexpr int kAccStages = OTIF_E12_ACC, kE1Slots = OTIF_E12_E1SLOTS;
    constexpr uint32_t kE1Col = kAccStages * 2 * 64;
    // TS: two im2col buffers of KT x 16 columns (K = 32 fp16 per row) after the E1 slots
    constexpr uint32_t kA1Col = kE1Col + kE1Slots * 32 * KT;
    static_assert(kA1Col + (OTIF_E12_TS ? 2 * 16 * KT : 0) <= 512, "TMEM budget");
    extern __shared__ __align__(1024) uint8_t smem[];
    const int warp = threadIdx.x >> 5;
    const int lane = threadIdx.x & 31;
    constexpr int N2 = 64;
    constexpr int MT = 2;
    constexpr int P = 128 * KT;
    constexpr uint32_t kW2Bytes = 9 * 4 * N2 * 16;     // 36,864
    constexpr uint32_t kW1Bytes = 4 * 32 * 16;         // 2,048
    constexpr uint32_t kA1Bytes = KT * 4 * 128 * 16;   // one plane's im2col rows
    constexpr uint32_t kPlaneBytes = P * 64;           // one plane's E1 activations (E2's A)
    const uint32_t slab_bytes = (uint32_t)p.slab_rows * p.slab_pitch;

    uint8_t *w2_s = smem;
    uint8_t *w1_s = w2_s + kW2Bytes;
    uint8_t *a1_s = w1_s + kW1Bytes;
    uint8_t *a2_s = a1_s + (OTIF_E12_TS ? (size_t)0 : (size_t)p.na1 * kA1Bytes);
    uint8_t *slab_s = a2_s + (size_t)p.np * kPlaneBytes;
    uint64_t *bars = reinterpret_cast<uint64_t *>(slab_s + 2 * (size_t)slab_bytes);
    uint64_t *slab_full = bars, *slab_empty = bars + 2;
    uint64_t *a1_full = bars + 4, *a1_empty = bars + 6;
    uint64_t *e1_full = bars + 8, *e1_empty = bars + 12;           // up to 4 slots each
    uint64_t *a2_full = bars + 16, *a2_empty = a2_full + kE12MaxPlaneBufs;
    uint64_t *acc_full = a2_empty + kE12MaxPlaneBufs, *acc_empty = acc_full + 2;
    uint32_t *tmem_slot = reinterpret_cast<uint32_t *>(acc_empty + 2);
    float *s_b1 = reinterpret_cast<float *>(tmem_slot + 4);
    float *s_b2 = s_b1 + 32;
    int &s_e12_done = *reinterpret_cast<int *>(s_b2 + 64);   // E2 epilogue drained its last tile

    // ---- prologue: barriers, TMEM, resident weights, slab pads = 128 ----
    if (threadIdx.x == 0) {
        for (int i = 0; i < 2; i++) {
            mbar_init(&slab_full[i], 1); mbar_init(&slab_empty[i], 256);
            mbar_init(&a1_full[i], 256); mbar_init(&a1_empty[i], 1);
            mbar_init(&acc_full[i], 1); mbar_init(&acc_empty[i], 128);
        }
        for (int i = 0; i < kE1Slots; i++) { mbar_init(&e1_full[i], 1); mbar_init(&e1_empty[i], 256); }
        for (int i = 0; i < kE12MaxPlaneBufs; i++) { mbar_init(&a2_full[i], 256); mbar_init(&a2_empty[i], 1); }
        fence_barrier_init();
    }
    if (warp == 2) tmem_alloc(tmem_slot, 512);
    for (uint32_t i = threadIdx.x; i < kW2Bytes / 16; i += blockDim.x)
        reinterpret_cast<uint4 *>(w2_s)[i] = reinterpret_cast<const uint4 *>(p.wt2)[i];
    for (uint32_t i = threadIdx.x; i < kW1Bytes / 16; i += blockDim.x)
        reinterpret_cast<uint4 *>(w1_s)[i] = reinterpret_cast<const uint4 *>(p.wt1)[i];
    for (uint32_t i = threadIdx.x; i < 2 * slab_bytes / 16; i += blockDim.x)
        reinterpret_cast<uint4 *>(slab_s)[i] = make_uint4(0x80808080u, 0x80808080u, 0x80808080u, 0x80808080u);
    if (threadIdx.x < N2) s_b2[threadIdx.x] = p.b2[threadIdx.x];
    if (threadIdx.x == 0) s_e12_done = 0;
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");  // resident weights -> tensor core
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem_base = *tmem_slot;
    const uint32_t rows_per_frame = (uint32_t)p.h2 + 1;   // plane rows per frame (row 0 = pad)
    E12_TR_DECL

    if (warp == 0) {
        // ===== slab loader =====
        uint32_t sb = 0, sp = 0;
        for (int tile = blockIdx.x; tile < p.ntiles; tile += gridDim.x) {
            const uint32_t q0 = (uint32_t)tile * (128 * MT);
            const uint32_t g0 = fdiv(q0, p.div_pitch);
            E12_WAIT_SLEEP(&slab_empty[sb], sp ^ 1);
            uint8_t *slab = slab_s + (size_t)sb * slab_bytes;
            // slab row s: s = 0 -> image row 4(i0-1)-1 of plane row g0; s >= 1 -> plane row g0 + (s-1)/4, k = (s-1)%4
            uint32_t my_bytes = 0;
            for (int s = lane; s < p.slab_rows; s += 32) {
                const uint32_t g = s == 0 ? g0 : g0 + (s - 1) / 4;
                const int k = s == 0 ? -1 : (s - 1) % 4;
                const uint32_t f = fdiv(g, p.div_rpf);
                const int i = (int)(g - f * rows_per_frame);
                const int y = 4 * (i - 1) + k;
                if ((int)f < p.n && i >= 1 && y >= 0 && y < p.hp && !(E12_BITS & 64)) my_bytes += p.row_bytes;
            }
            if (p.bulk) {
#pragma unroll
                for (int o = 16; o >= 1; o >>= 1) my_bytes += __shfl_xor_sync(0xffffffffu, my_bytes, o);
                if (lane == 0 && my_bytes) mbar_expect_tx(&slab_full[sb], my_bytes);
                __syncwarp();
            }
            for (int s = lane; s < p.slab_rows; s += 32) {
                const uint32_t g = s == 0 ? g0 : g0 + (s - 1) / 4;
                const int k = s == 0 ? -1 : (s - 1) % 4;
                const uint32_t f = fdiv(g, p.div_rpf);
                const int i = (int)(g - f * rows_per_frame);
                const int y = 4 * (i - 1) + k;
                uint8_t *dst = slab + (size_t)s * p.slab_pitch;
                if ((int)f < p.n && i >= 1 && y >= 0 && y < p.hp && !(E12_BITS & 64)) {   // 64: timing experiment
                    const uint8_t *src = p.img + ((size_t)f * p.hp + y) * p.row_bytes;
                    if (p.bulk) {
                        bulk_g2s(dst + 16, src, p.row_bytes, &slab_full[sb]);
                    } else {
#pragma unroll 1
                        for (int b = 0; b < p.row_bytes; b++) dst[16 + b] = __ldg(src + b);
                    }
                } else {
#pragma unroll 1
                    for (int b = 0; b < p.slab_pitch; b += 16)
                        *reinterpret_cast<uint4 *>(dst + b) = make_uint4(0x80808080u, 0x80808080u, 0x80808080u, 0x80808080u);
                }
            }
            __threadfence_block();
            __syncwarp();
            if (lane == 0) mbar_arrive(&slab_full[sb]);
            if (++sb == 2) { sb = 0; sp ^= 1; }
        }
    } else if (warp == 1) {
        // ===== E1 MMA issuer (whole warp, elected lane issues): one plane job per hand-off =====
        const uint32_t idesc1 = umma_idesc_f16(128, 32);
        const uint64_t a1d = umma_desc(smem_u32(a1_s), 2048, 128);
        const uint64_t w1d = umma_desc(smem_u32(w1_s), 512, 128);
        uint32_t J = 0;
        for (int tile = blockIdx.x; tile < p.ntiles; tile += gridDim.x) {
            for (int g = 0; g < 4; g++, J++) {
                const uint32_t s1 = (uint32_t)p.na1 == 1 ? 0 : (J & 1);
                const uint32_t ph1 = (uint32_t)p.na1 == 1 ? (J & 1) : ((J >> 1) & 1);
                mbar_wait(&a1_full[s1], ph1);
                E12_TR(0, 0);
                mbar_wait(&e1_empty[J % kE1Slots], ((J / kE1Slots) & 1) ^ 1);
                E12_TR(1, 0);
                tc_fence_after();
                const uint32_t d = tmem_base + kE1Col + (J % kE1Slots) * (32 * KT);
#pragma unroll
                for (int k = 0; k < KT; k++)
#pragma unroll
                    for (int s = 0; s < 2; s++) {
#if OTIF_E12_TS
                        umma_ts_warp(d + k * 32, tmem_base + kA1Col + s1 * 16 * KT + k * 16 + s * 8,
                                     w1d + ((2 * s * 512) >> 4), idesc1, s);
#else
                        umma_bf16_warp(d + k * 32, a1d + ((s1 * kA1Bytes + k * 8192 + 2 * s * 2048) >> 4),
                                           w1d + ((2 * s * 512) >> 4), idesc1, s);
#endif
                    }
                umma_commit_warp(&a1_empty[s1]);
                umma_commit_warp(&e1_full[J % kE1Slots]);
                E12_TR(2, 0);
            }
        }
        E12_TR_DUMP("E1MMA a1full e1empty issued", 3);
    } else if (warp == 3) {
        // ===== E2 MMA issuer (whole warp, elected lane issues) =====
        const uint32_t idesc2 = umma_idesc_bf16(128, N2);
        const uint64_t a2d = umma_desc(smem_u32(a2_s), P * 16, 128);
        const uint64_t w2d = umma_desc(smem_u32(w2_s), N2 * 16, 128);
        uint32_t pb = 0, pp = 0, acc = 0, accp = 0, J = 0;
        for (int tile = blockIdx.x; tile < p.ntiles; tile += gridDim.x) {
            mbar_wait(&acc_empty[acc], accp ^ 1);
            tc_fence_after();
            const uint32_t d = tmem_base + acc * (MT * N2);
            int pos = 0;
            for (int g = 0; g < 4; g++, J++) {
                E12_TR(0, 0);
                mbar_wait(&a2_full[pb], pp);
                E12_TR(1, 0);
                tc_fence_after();
                const uint64_t a = a2d + ((pb * kPlaneBytes) >> 4);
                const int ntaps = (E12_BITS & 8) ? 1 : p.group_ntaps[g];   // trace & 8: timing experiment
#pragma unroll 1
                for (int t = 0; t < ntaps; t++, pos++) {
                    const uint64_t at = a + p.group_shift[g][t];          // +16 B per pixel of shift
                    const uint64_t bt = w2d + ((pos * (4 * N2 * 16)) >> 4);
#pragma unroll
                    for (int s = 0; s < 2; s++)
#pragma unroll
                        for (int mm = 0; mm < MT; mm++)
                            umma_bf16_warp(d + mm * N2, at + ((2 * s * P * 16 + mm * 2048) >> 4), bt + ((2 * s * N2 * 16) >> 4),
                                           idesc2, (g == 0 && t == 0 && s == 0) ? 0u : 1u);
                }
                umma_commit_warp(&a2_empty[pb]);
                E12_TR(2, 0);
                if (++pb == (uint32_t)p.np) { pb = 0; pp ^= 1; }
            }
            umma_commit_warp(&acc_full[acc]);
            if (++acc == kAccStages) { acc = 0; accp ^= 1; }
        }
        E12_TR_DUMP("E2MMA start a2full issued", 3);
    } else if (warp >= 4 && warp < 12) {
        // ===== gather (2 warpgroups, alternate E1 M tiles): one im2col row per thread =====
        const int wg = (warp - 4) >> 2;
        const int row = (threadIdx.x - 128) & 127;
        uint32_t J = 0, sb = 0, sp = 0;
        for (int tile = blockIdx.x; tile < p.ntiles; tile += gridDim.x) {
            const uint32_t q0 = (uint32_t)tile * (128 * MT);
            const uint32_t g0 = fdiv(q0, p.div_pitch);
            uint32_t vm[KT], of[KT];
#pragma unroll
            for (int k = 0; k < KT; k++) e12_decode(p, q0 + k * 128 + row, g0, vm[k], of[k]);
            E12_WAIT_SLEEP(&slab_full[sb], sp);
            const uint8_t *slab = slab_s + (size_t)sb * slab_bytes;
#pragma unroll 1
            for (int g = 0; g < 4; g++, J++) {
                const int rp = g >> 1, cp = g & 1;
                const uint32_t s1 = (uint32_t)p.na1 == 1 ? 0 : (J & 1);
                const uint32_t ph1 = (uint32_t)p.na1 == 1 ? (J & 1) : ((J >> 1) & 1);
                E12_TR(0, 0);
                E12_WAIT_CHAIN(&a1_empty[s1], ph1 ^ 1);
                E12_TR(1, 0);
                {
#if OTIF_E12_GATHER2 && !OTIF_E12_TS
                    // both of this thread's rows (sub-tiles k0 and k0 + 2) built together: their
                    // slab loads and conversions interleave (the gather is the critical role,
                    // profiles/r02p_e12_source.md)
                    const int k0 = (int)((wg - J * KT) & 1);
                    const bool two = k0 + 2 < KT;
                    uint32_t va = vm[0], oa = of[0], vb = vm[KT - 1], ob = of[KT - 1];
#pragma unroll
                    for (int i = 1; i < KT; i++)
                        if (k0 == i) { va = vm[i]; oa = of[i]; }
                    if (KT == 4 && k0 == 0) { vb = vm[2]; ob = of[2]; }
                    uint32_t wa[16], wb[16];
                    e12_im2col_row(p, slab, (va >> g) & 1, oa, rp, cp, wa);
                    e12_im2col_row(p, slab, two ? ((vb >> g) & 1) : 0u, ob, rp, cp, wb);
                    {
                        uint8_t *dst = a1_s + s1 * kA1Bytes + k0 * 8192 + row * 16;
#pragma unroll
                        for (int c = 0; c < 4; c++)
                            *reinterpret_cast<uint4 *>(dst + c * 2048) = make_uint4(wa[4 * c], wa[4 * c + 1], wa[4 * c + 2], wa[4 * c + 3]);
                        if (two) {
#pragma unroll
                            for (int c = 0; c < 4; c++)
                                *reinterpret_cast<uint4 *>(dst + 2 * 8192 + c * 2048) =
                                    make_uint4(wb[4 * c], wb[4 * c + 1], wb[4 * c + 2], wb[4 * c + 3]);
                        }
                    }
                    if (false)
#endif
                    // rolled loop over this warpgroup's k sub-tiles (code size: the kernel is
                    // instruction-cache bound, see the header)
#pragma unroll 1
                    for (int k = (int)((wg - J * KT) & 1); k < KT; k += 2) {
                        uint32_t vmk = vm[0], ofk = of[0];
#pragma unroll
                        for (int i = 1; i < KT; i++)
                            if (k == i) { vmk = vm[i]; ofk = of[i]; }
                        uint32_t wv[16];
                        e12_im2col_row(p, slab, (vmk >> g) & 1, ofk, rp, cp, wv);
#if OTIF_E12_TS
                        // this warp's 32 TMEM lanes = its 32 rows of sub-tile k (lane = row)
                        tmem_st16(tmem_base + ((uint32_t)(row & ~31) << 16) + kA1Col + s1 * 16 * KT + k * 16, wv);
#else
                        uint8_t *dst = a1_s + s1 * kA1Bytes + k * 8192 + row * 16;
#pragma unroll
                        for (int c = 0; c < 4; c++)
                            *reinterpret_cast<uint4 *>(dst + c * 2048) = make_uint4(wv[4 * c], wv[4 * c + 1], wv[4 * c + 2], wv[4 * c + 3]);
#endif
                    }
                }
#if OTIF_E12_TS
                tmem_wait_st();
                tc_fence_before();
#else
                asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
#endif
                mbar_arrive(&a1_full[s1]);
                E12_TR(2, 0);
            }
            mbar_arrive(&slab_empty[sb]);
            if (++sb == 2) { sb = 0; sp ^= 1; }
        }
        E12_TR_DUMP("GATH start a1empty arrived", 3);
    } else if (warp >= 12 && warp < 20) {
        // ===== E1 epilogue (2 warpgroups, alternate E1 M tiles): TMEM -> ReLU, bf16 -> plane
        // buffer (E2's A operand).  The accumulator already holds 2^(s+7) (E1 sum + bias);
        // rounding to bf16 commutes with that power-of-two scale, which E2's weights undo.
        // Positions without an E1 pixel have an all-zero A row, hence exactly zero here.
        const int wg = (warp - 12) >> 2;
        const int row = (threadIdx.x - 384) & 127;
        const int quarter = warp & 3;
        uint32_t J = 0, pb = 0, pp = 0;
        for (int tile = blockIdx.x; tile < p.ntiles; tile += gridDim.x) {
#pragma unroll 1
            for (int g = 0; g < 4; g++, J++) {
                E12_WAIT_CHAIN(&a2_empty[pb], pp ^ 1);
                E12_TR(0, 0);
                mbar_wait(&e1_full[J % kE1Slots], (J / kE1Slots) & 1);
                E12_TR(1, 0);
                tc_fence_after();
                uint8_t *plane = a2_s + pb * kPlaneBytes;
                const uint32_t tacc = tmem_base + ((uint32_t)(quarter * 32) << 16) + kE1Col + (J % kE1Slots) * (32 * KT);
#pragma unroll 1
                for (int k = (int)((wg - J * KT) & 1); k < KT; k += 2) {
                    if (E12_BITS & 32) continue;   // 32: timing experiment
                    uint32_t v[32];
                    tmem_ld32(tacc + k * 32, v);
                    uint32_t pk[16];
#pragma unroll
                    for (int j = 0; j < 16; j++) pk[j] = pack_bf16x2_relu(__uint_as_float(v[2 * j]), __uint_as_float(v[2 * j + 1]));
                    uint8_t *dst = plane + (size_t)(k * 128 + row) * 16;
#pragma unroll
                    for (int c = 0; c < 4; c++)
                        *reinterpret_cast<uint4 *>(dst + (size_t)c * P * 16) =
                            make_uint4(pk[4 * c], pk[4 * c + 1], pk[4 * c + 2], pk[4 * c + 3]);
                }
                tc_fence_before();
                mbar_arrive(&e1_empty[J % kE1Slots]);
                asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
                mbar_arrive(&a2_full[pb]);
                E12_TR(2, 0);
                if (++pb == (uint32_t)p.np) { pb = 0; pp ^= 1; }
            }
        }
        E12_TR_DUMP("E1EP a2empty e1full arrived", 3);
    } else if (warp >= 24) {
        // ===== fused pack of the previous batch (packjob.cuh) until the E2 epilogue is done =====
        if (p.pj) pj_drain_warp<OTIF_PJ_UNROLL>(p.pj, &s_e12_done, lane);
    } else if (warp >= 20) {
        // ===== E2 epilogue: TMEM -> bias, ReLU, bf16 -> E3's input layout =====
        const int row = threadIdx.x - 640;
        const int quarter = warp & 3;
        uint32_t acc = 0, accp = 0;
        for (int tile = blockIdx.x; tile < p.ntiles; tile += gridDim.x) {
            E12_WAIT_SLEEP(&acc_full[acc], accp);
            tc_fence_after();
#pragma unroll 1
            for (int mm = 0; mm < MT; mm++) {
                const uint32_t q = (uint32_t)tile * (128 * MT) + mm * 128 + row;
                const uint32_t f = fdiv(q, p.div_fstride);
                const uint32_t r = q - f * p.fstride;
                const uint32_t oy = fdiv(r, p.div_pitch);
                const int ox = (int)(r - oy * (uint32_t)p.pitch);
                const bool valid = q < p.mtot && (int)oy < p.h2 && ox < p.w2;
                int plane = 0;
                const int64_t L = layout_pixel(p.out_kind, p.out_pitch, p.out_fstride, (int)f, (int)oy, ox, plane);
                const uint32_t taddr = tmem_base + ((uint32_t)(quarter * 32) << 16) + acc * (MT * N2) + mm * N2;
                // this row's first 8-channel chunk; chunks are lcap * 16 bytes apart
                uint8_t *const row_out = p.out + ((int64_t)plane * p.out_c8 * p.out_lcap + L) * 16;
                const int64_t chunk_stride = p.out_lcap * 16;
#pragma unroll
                for (int cc = 0; cc < N2 / 32; cc++) {
                    uint32_t v[32];
                    tmem_ld32(taddr + cc * 32, v);
                    if (valid && !(E12_BITS & 16)) {   // 16: timing experiment
                        uint32_t pk[16];
#pragma unroll
                        for (int j = 0; j < 16; j++)
                            pk[j] = pack_bf16x2_relu(__uint_as_float(v[2 * j]) + s_b2[cc * 32 + 2 * j],
                                                     __uint_as_float(v[2 * j + 1]) + s_b2[cc * 32 + 2 * j + 1]);
#pragma unroll
                        for (int c = 0; c < 4; c++)
                            *reinterpret_cast<uint4 *>(row_out + (cc * 4 + c) * chunk_stride) =
                                make_uint4(pk[4 * c], pk[4 * c + 1], pk[4 * c + 2], pk[4 * c + 3]);
                    }
                }
            }
            tc_fence_before();
            mbar_arrive(&acc_empty[acc]);
            if (++acc == kAccStages) { acc = 0; accp ^= 1; }
        }
        if (threadIdx.x == 640) *(volatile int *)&s_e12_done = 1;
    }
    __syncwarp();
    tc_fence_before();
    __syncthreads();
    if (warp == 2) {
        tc_fence_after();
        tmem_dealloc(tmem_base, 512);
    }
}

#if OTIF_E12B_BUILD
// ---------------------------------------------------------------------------
// E1 fused into E2, "band" variant (e12b).  Same arithmetic as e12_umma_kernel (exact fp16
// im2col rows u - 128 against w * 2^s, bias folded into K, E2 weights * 2^-(s+7)), but the
// unit of work is a BAND: R consecutive E2 output rows of one frame (M = 256 positions,
// R * pitch <= 256 valid) with ALL FOUR parity planes of its E1 input computed at once
// (4 x PB plane-buffer rows, PB >= 256 + pitch + 1).  Per band there are four hand-offs
// (gather -> E1 MMA -> E1 epilogue -> E2 MMA) instead of sixteen per 256-position tile,
// and consecutive bands of a frame share image rows through a ring (only 4R new image
// rows per band are loaded).  Buffers are single-stage (A1 im2col 256 PB B, planes
// 256 PB B, E1 accumulators PB TMEM columns, E2 accumulators 128 columns); E2's weights
// stream through a 3-stage ring of per-tap stages.  Roles (768 threads): warp 0 image-row
// loader, warp 1 E1 MMA, warp 2 TMEM allocator then weight-stage loader, warp 3 E2 MMA,
// warps 4-11 gather (5 im2col rows per thread), 12-19 E1 epilogue (alternate 128-row
// sub-tiles), 20-23 E2 epilogue.
// ---------------------------------------------------------------------------
struct E12bParams {
    const uint8_t *img;         // u8 [n, hp, wp, 3]
    int n, hp, wp, row_bytes;
    int h1, w1, h2, w2, pitch;  // E1 / E2 output sizes; pitch = w2 + 1 (E2-input plane layout)
    int R;                      // E2 output rows per band
    int nbpf;                   // bands per frame = ceil(h2 / R)
    int njobs;                  // n * nbpf
    int PB;                     // plane-buffer rows (multiple of 32)
    int D;                      // (PB - 1) / pitch: plane rows spanned beyond the band's first
    int NR;                     // image rows per band = 4 D + 5
    int RC;                     // image-row ring capacity (rows) = 2 NR
    int ring_pitch;             // bytes per ring row (16-B left pad, row, right pad)
    int bulk;                   // rows may be bulk-copied (16-B aligned)
    FastDiv div_pitch, div_PB, div_RC;
    const uint16_t *wt1;        // fp16 [4 chunks][32 n][8] (as e12)
    const uint16_t *wt2;        // bf16 [9 taps in loop order][4 chunks][64 n][8] (as e12)
    const float *b2;
    int group_ntaps[4], group_shift[4][9];
    int out_kind;
    uint8_t *out;
    int64_t out_lcap;
    int out_c8, out_pitch;
    int64_t out_fstride;
};

constexpr int kE12bThreads = 768;
constexpr int kE12bW2Stages = 3;

// job index -> (frame, band) and whether it continues the previous job's frame band
__device__ __forceinline__ void e12b_job(const E12bParams &p, int j, int &f, int &b) {
    f = j / p.nbpf;
    b = j - f * p.nbpf;
}

// One E1 im2col row (fp16, K = 32 with the bias slots), as e12_im2col_row, from three
// ring rows (image rows 2y-1, 2y, 2y+1) at byte offset `off` (column 2x-1, can be the pad)
__device__ __forceinline__ void e12b_im2col_row(const uint8_t *r0, const uint8_t *r1, const uint8_t *r2, uint32_t off,
                                                uint32_t (&wv)[16]) {
    const uint32_t sh = (off & 3) * 8;
    const uint8_t *rows[3] = {r0, r1, r2};
#pragma unroll
    for (int kh = 0; kh < 3; kh++) {
        const uint32_t *wp = reinterpret_cast<const uint32_t *>(rows[kh] + (off & ~3u));
        const uint32_t w0 = wp[0], w1 = wp[1], w2 = wp[2];
        const uint32_t a0 = __funnelshift_r(w0, w1, sh), a1 = __funnelshift_r(w1, w2, sh);
        wv[5 * kh + 0] = sub_f16x2(__byte_perm(a0, 0x64646464u, 0x4140), 0x64806480u);
        wv[5 * kh + 1] = sub_f16x2(__byte_perm(a0, 0x64646464u, 0x4342), 0x64806480u);
        wv[5 * kh + 2] = sub_f16x2(__byte_perm(a1, 0x64646464u, 0x4140), 0x64806480u);
        wv[5 * kh + 3] = sub_f16x2(__byte_perm(a1, 0x64646464u, 0x4342), 0x64806480u);
        wv[5 * kh + 4] = sub_f16x2(0x64006400u | ((w2 >> sh) & 0xFFu), 0x63006480u);
    }
    wv[15] = 0;
}

#ifdef OTIF_E12_TRACE_BUILD   // timeline of CTA 0, bands 20..35 (debug builds only)
#define E12B_TR_DECL const bool trb = blockIdx.x == 0 && (threadIdx.x & 31) == 0; long long tb[3][16]; const long long tb0 = clock64();
#define E12B_TR(slot) do { if (trb && k >= 20 && k < 36) tb[slot][k - 20] = clock64() - tb0; } while (0)
#define E12B_TR_DUMP(name) do { if (trb && (threadIdx.x == 0 || threadIdx.x == 32 || threadIdx.x == 96 || threadIdx.x == 128 || threadIdx.x == 384 || threadIdx.x == 640)) \
    for (int q_ = 0; q_ < 16 && q_ + 20 < (j1 - j0); q_++) printf("%s k=%2d %8lld %8lld %8lld\n", name, q_ + 20, tb[0][q_], tb[1][q_], tb[2][q_]); } while (0)
#else
#define E12B_TR_DECL
#define E12B_TR(slot) do {} while (0)
#define E12B_TR_DUMP(name) do {} while (0)
#endif
__global__ void __launch_bounds__(kE12bThreads, 1) e12b_umma_kernel(const __grid_constant__ E12bParams p) {
    extern __shared__ __align__(1024) uint8_t smem[];
    const int warp = threadIdx.x >> 5;
    const int lane = threadIdx.x & 31;
    constexpr int N2 = 64;
    constexpr uint32_t kW2Stage = 4 * N2 * 16;         // one tap: [4 chunks][64 n][8] bf16 = 4 KB
    constexpr uint32_t kW1Bytes = 4 * 32 * 16;
    const int PB = p.PB;
    const int nsub = 4 * PB / 128;                     // E1 M sub-tiles per band
    const uint32_t a1_bytes = (uint32_t)nsub * 8192;   // [sub][chunk][128 rows][16 B]
    const uint32_t pl_bytes = (uint32_t)PB * 64;       // one plane: [chunk][PB rows][16 B]
    const uint32_t ring_bytes = (uint32_t)p.RC * p.ring_pitch;

    uint8_t *a1_s = smem;
    uint8_t *pl_s = a1_s + a1_bytes;
    uint8_t *w2_s = pl_s + 4 * pl_bytes;
    uint8_t *w1_s = w2_s + kE12bW2Stages * kW2Stage;
    uint8_t *ring_s = w1_s + kW1Bytes;
    uint64_t *bars = reinterpret_cast<uint64_t *>(ring_s + ring_bytes);
    uint64_t *ring_full = bars, *ring_empty = bars + 2;
    uint64_t *w2_full = bars + 4, *w2_empty = w2_full + kE12bW2Stages;
    uint64_t *a1_full = w2_empty + kE12bW2Stages, *a1_empty = a1_full + 1;
    uint64_t *e1_full = a1_empty + 1, *e1_empty = e1_full + 1;
    uint64_t *pl_full = e1_empty + 1, *pl_empty = pl_full + 1;
    uint64_t *acc_full = pl_empty + 1, *acc_empty = acc_full + 1;
    uint32_t *tmem_slot = reinterpret_cast<uint32_t *>(acc_empty + 1);
    float *s_b2 = reinterpret_cast<float *>(tmem_slot + 4);

    if (threadIdx.x == 0) {
        for (int i = 0; i < 2; i++) { mbar_init(&ring_full[i], 1); mbar_init(&ring_empty[i], 256); }
        for (int i = 0; i < kE12bW2Stages; i++) { mbar_init(&w2_full[i], 1); mbar_init(&w2_empty[i], 1); }
        mbar_init(a1_full, 256); mbar_init(a1_empty, 1);
        mbar_init(e1_full, 1); mbar_init(e1_empty, 256);
        mbar_init(pl_full, 256); mbar_init(pl_empty, 1);
        mbar_init(acc_full, 1); mbar_init(acc_empty, 128);
        fence_barrier_init();
    }
    if (warp == 2) tmem_alloc(tmem_slot, 512);
    for (uint32_t i = threadIdx.x; i < kW1Bytes / 16; i += blockDim.x)
        reinterpret_cast<uint4 *>(w1_s)[i] = reinterpret_cast<const uint4 *>(p.wt1)[i];
    // ring: every byte 128 (x = 0): the pads around each row are never written again
    for (uint32_t i = threadIdx.x; i < ring_bytes / 16; i += blockDim.x)
        reinterpret_cast<uint4 *>(ring_s)[i] = make_uint4(0x80808080u, 0x80808080u, 0x80808080u, 0x80808080u);
    if (threadIdx.x < N2) s_b2[threadIdx.x] = p.b2[threadIdx.x];
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem_base = *tmem_slot;
    constexpr uint32_t kE1Col = 128;                  // E2 accumulators: columns [0, 128)

    // contiguous job range of this CTA (consecutive bands of a frame share image rows)
    const int j0 = (int)((int64_t)blockIdx.x * p.njobs / gridDim.x);
    const int j1 = (int)((int64_t)(blockIdx.x + 1) * p.njobs / gridDim.x);
    E12B_TR_DECL

    if (warp == 0) {
        // ===== loader: image rows of each band into the ring =====
        int seq_base = -p.NR, pf = -1, pb = -1;
        for (int j = j0, k = 0; j < j1; j++, k++) {
            int f, b;
            e12b_job(p, j, f, b);
            const bool cont = (f == pf && b == pb + 1);
            const int fresh0 = cont ? p.NR - 4 * p.R : 0;   // first band-relative row to load
            seq_base = cont ? seq_base + 4 * p.R : seq_base + p.NR;
            pf = f; pb = b;
            const int Y0 = 4 * b * p.R - 5;
            E12B_TR(0);
            // band k-2's rows are free once its gather is done
            mbar_wait(&ring_empty[k & 1], ((k >> 1) & 1) ^ 1);
            E12B_TR(1);
            uint32_t my_bytes = 0;
            for (int i = fresh0 + lane; i < p.NR; i += 32) {
                const int y = Y0 + i;
                if (y >= 0 && y < p.hp) my_bytes += p.row_bytes;
            }
            if (p.bulk) {
#pragma unroll
                for (int o = 16; o >= 1; o >>= 1) my_bytes += __shfl_xor_sync(0xffffffffu, my_bytes, o);
                if (lane == 0 && my_bytes) mbar_expect_tx(&ring_full[k & 1], my_bytes);
                __syncwarp();
            }
            for (int i = fresh0 + lane; i < p.NR; i += 32) {
                const int y = Y0 + i;
                const uint32_t slot = (uint32_t)(seq_base + i) - fdiv((uint32_t)(seq_base + i), p.div_RC) * p.RC;
                uint8_t *dst = ring_s + (size_t)slot * p.ring_pitch + 16;
                if (y >= 0 && y < p.hp) {
                    const uint8_t *src = p.img + ((size_t)f * p.hp + y) * p.row_bytes;
                    if (p.bulk) {
                        bulk_g2s(dst, src, p.row_bytes, &ring_full[k & 1]);
                    } else {
#pragma unroll 1
                        for (int q = 0; q < p.row_bytes; q++) dst[q] = __ldg(src + q);
                    }
                } else {
#pragma unroll 1
                    for (int q = 0; q < p.row_bytes; q += 4)
                        *reinterpret_cast<uint32_t *>(dst + q) = 0x80808080u;
                }
            }
            __threadfence_block();
            __syncwarp();
            if (lane == 0) mbar_arrive(&ring_full[k & 1]);
            E12B_TR(2);
        }
        E12B_TR_DUMP("LOAD");
    } else if (warp == 2) {
        // ===== weight loader (after the TMEM allocation): the nine E2 tap stages per band =====
        if (lane == 0) {
            uint32_t ws = 0, wph = 0;
            for (int j = j0; j < j1; j++) {
#pragma unroll 1
                for (int t = 0; t < 9; t++) {
                    mbar_wait(&w2_empty[ws], wph ^ 1);
                    mbar_arrive_expect_tx(&w2_full[ws], kW2Stage);
                    bulk_g2s(w2_s + ws * kW2Stage, reinterpret_cast<const uint8_t *>(p.wt2) + t * kW2Stage, kW2Stage,
                             &w2_full[ws]);
                    if (++ws == kE12bW2Stages) { ws = 0; wph ^= 1; }
                }
            }
        }
    } else if (warp == 1) {
        // ===== E1 MMA issuer (whole warp, elected lane): nsub x 2 MMAs per band =====
        const uint32_t idesc1 = umma_idesc_f16(128, 32);
        const uint64_t a1d = umma_desc(smem_u32(a1_s), 2048, 128);
        const uint64_t w1d = umma_desc(smem_u32(w1_s), 512, 128);
        for (int j = j0, k = 0; j < j1; j++, k++) {
            mbar_wait(a1_full, k & 1);
            E12B_TR(0);
            mbar_wait(e1_empty, (k & 1) ^ 1);
            E12B_TR(1);
            tc_fence_after();
#pragma unroll 1
            for (int m = 0; m < nsub; m++)
#pragma unroll
                for (int s = 0; s < 2; s++)
                    umma_bf16_warp(tmem_base + kE1Col + m * 32, a1d + ((m * 8192 + 2 * s * 2048) >> 4),
                                   w1d + ((2 * s * 512) >> 4), idesc1, s);
            umma_commit_warp(a1_empty);
            umma_commit_warp(e1_full);
            E12B_TR(2);
        }
        E12B_TR_DUMP("E1MMA");
    } else if (warp == 3) {
        // ===== E2 MMA issuer: 9 taps x 2 K halves x 2 M sub-tiles per band =====
        const uint32_t idesc2 = umma_idesc_bf16(128, N2);
        const uint64_t pld = umma_desc(smem_u32(pl_s), PB * 16, 128);
        const uint64_t w2d = umma_desc(smem_u32(w2_s), N2 * 16, 128);
        uint32_t ws = 0, wph = 0;
        for (int j = j0, k = 0; j < j1; j++, k++) {
            mbar_wait(pl_full, k & 1);
            E12B_TR(0);
            mbar_wait(acc_empty, (k & 1) ^ 1);
            E12B_TR(1);
            tc_fence_after();
            int pos = 0;
#pragma unroll 1
            for (int g = 0; g < 4; g++) {
                const uint64_t a = pld + ((g * pl_bytes) >> 4);
#pragma unroll 1
                for (int t = 0; t < p.group_ntaps[g]; t++, pos++) {
                    mbar_wait(&w2_full[ws], wph);
                    tc_fence_after();
                    const uint64_t at = a + p.group_shift[g][t];          // +16 B per position
                    const uint64_t bt = w2d + ((ws * kW2Stage) >> 4);
#pragma unroll
                    for (int s = 0; s < 2; s++)
#pragma unroll
                        for (int mm = 0; mm < 2; mm++)
                            umma_bf16_warp(tmem_base + mm * N2, at + ((2 * s * PB * 16 + mm * 2048) >> 4),
                                           bt + ((2 * s * N2 * 16) >> 4), idesc2, (pos == 0 && s == 0) ? 0u : 1u);
                    umma_commit_warp(&w2_empty[ws]);
                    if (++ws == kE12bW2Stages) { ws = 0; wph ^= 1; }
                }
            }
            umma_commit_warp(pl_empty);
            umma_commit_warp(acc_full);
            E12B_TR(2);
        }
        E12B_TR_DUMP("E2MMA");
    } else if (warp >= 4 && warp < 12) {
        // ===== gather: the band's 4 x PB im2col rows (plane g = r / PB, row j = r % PB) =====
        const int gt = threadIdx.x - 128;            // 0..255
        int seq_base = -p.NR, pf = -1, pb = -1;
        for (int j = j0, k = 0; j < j1; j++, k++) {
            int f, b;
            e12b_job(p, j, f, b);
            const bool cont = (f == pf && b == pb + 1);
            seq_base = cont ? seq_base + 4 * p.R : seq_base + p.NR;
            pf = f; pb = b;
            const int oy0 = b * p.R;
            const int Y0 = 4 * oy0 - 5;
            mbar_wait(&ring_full[k & 1], (k >> 1) & 1);
            E12B_TR(0);
            mbar_wait(a1_empty, (k & 1) ^ 1);
            E12B_TR(1);
#pragma unroll 1
            for (int r = gt; r < 4 * PB; r += 256) {
                const uint32_t g = fdiv((uint32_t)r, p.div_PB);
                const uint32_t jj = (uint32_t)r - g * (uint32_t)PB;
                const uint32_t pp = (uint32_t)(oy0 * p.pitch) + jj;
                const uint32_t pr = fdiv(pp, p.div_pitch);
                const uint32_t pc = pp - pr * (uint32_t)p.pitch;
                const int rp = (int)(g >> 1), cp = (int)(g & 1);
                const int y = 2 * ((int)pr - 1) + rp, x = 2 * ((int)pc - 1) + cp;
                const bool valid = pr >= 1 && (int)pr <= p.h2 && pc >= 1 && (int)pc <= p.w2 && y < p.h1 && x < p.w1;
                uint32_t wv[16];
                if (valid) {
                    const uint8_t *rr[3];
#pragma unroll
                    for (int kh = 0; kh < 3; kh++) {
                        const uint32_t s = (uint32_t)(seq_base + (2 * y - 1 + kh - Y0));
                        const uint32_t slot = s - fdiv(s, p.div_RC) * p.RC;
                        rr[kh] = ring_s + (size_t)slot * p.ring_pitch;
                    }
                    e12b_im2col_row(rr[0], rr[1], rr[2], (uint32_t)(6 * x + 13), wv);
                } else {
#pragma unroll
                    for (int q = 0; q < 16; q++) wv[q] = 0;
                }
                uint8_t *dst = a1_s + (size_t)(r >> 7) * 8192 + (r & 127) * 16;
#pragma unroll
                for (int c = 0; c < 4; c++)
                    *reinterpret_cast<uint4 *>(dst + c * 2048) = make_uint4(wv[4 * c], wv[4 * c + 1], wv[4 * c + 2], wv[4 * c + 3]);
            }
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
            mbar_arrive(a1_full);
            mbar_arrive(&ring_empty[k & 1]);
            E12B_TR(2);
        }
        E12B_TR_DUMP("GATH");
    } else if (warp >= 12 && warp < 20) {
        // ===== E1 epilogue: TMEM -> ReLU, bf16 -> plane buffers (E2's A operand) =====
        const int wg = (warp - 12) >> 2;
        const int quarter = warp & 3;
        const int lrow = quarter * 32 + lane;
        for (int j = j0, k = 0; j < j1; j++, k++) {
            mbar_wait(e1_full, k & 1);
            E12B_TR(0);
            mbar_wait(pl_empty, (k & 1) ^ 1);
            E12B_TR(1);
            tc_fence_after();
#pragma unroll 1
            for (int m = wg; m < nsub; m += 2) {
                uint32_t v[32];
                tmem_ld32(tmem_base + ((uint32_t)(quarter * 32) << 16) + kE1Col + m * 32, v);
                uint32_t pk[16];
#pragma unroll
                for (int q = 0; q < 16; q++) pk[q] = pack_bf16x2_relu(__uint_as_float(v[2 * q]), __uint_as_float(v[2 * q + 1]));
                const uint32_t r = (uint32_t)(m * 128 + lrow);
                const uint32_t g = fdiv(r, p.div_PB);
                const uint32_t jj = r - g * (uint32_t)PB;
                uint8_t *dst = pl_s + (size_t)g * pl_bytes + (size_t)jj * 16;
#pragma unroll
                for (int c = 0; c < 4; c++)
                    *reinterpret_cast<uint4 *>(dst + (size_t)c * PB * 16) =
                        make_uint4(pk[4 * c], pk[4 * c + 1], pk[4 * c + 2], pk[4 * c + 3]);
            }
            tc_fence_before();
            mbar_arrive(e1_empty);
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
            mbar_arrive(pl_full);
            E12B_TR(2);
        }
        E12B_TR_DUMP("E1EP");
    } else if (warp >= 20) {
        // ===== E2 epilogue: TMEM -> bias, ReLU, bf16 -> E3's input layout =====
        const int row = threadIdx.x - 640;
        const int quarter = warp & 3;
        for (int j = j0, k = 0; j < j1; j++, k++) {
            int f, b;
            e12b_job(p, j, f, b);
            const int oy0 = b * p.R;
            const int oy_end = min(oy0 + p.R, p.h2);
            E12B_TR(0);
            mbar_wait(acc_full, k & 1);
            E12B_TR(1);
            tc_fence_after();
#pragma unroll 1
            for (int mm = 0; mm < 2; mm++) {
                const uint32_t qr = (uint32_t)(oy0 * p.pitch + mm * 128 + row);
                const uint32_t oy = fdiv(qr, p.div_pitch);
                const int ox = (int)(qr - oy * (uint32_t)p.pitch);
                const bool valid = (int)oy < oy_end && ox < p.w2;
                int plane = 0;
                const int64_t L = layout_pixel(p.out_kind, p.out_pitch, p.out_fstride, f, (int)oy, ox, plane);
                const uint32_t taddr = tmem_base + ((uint32_t)(quarter * 32) << 16) + mm * N2;
                uint8_t *const row_out = p.out + ((int64_t)plane * p.out_c8 * p.out_lcap + L) * 16;
                const int64_t chunk_stride = p.out_lcap * 16;
#pragma unroll
                for (int cc = 0; cc < N2 / 32; cc++) {
                    uint32_t v[32];
                    tmem_ld32(taddr + cc * 32, v);
                    if (valid) {
                        uint32_t pk[16];
#pragma unroll
                        for (int q = 0; q < 16; q++)
                            pk[q] = pack_bf16x2_relu(__uint_as_float(v[2 * q]) + s_b2[cc * 32 + 2 * q],
                                                     __uint_as_float(v[2 * q + 1]) + s_b2[cc * 32 + 2 * q + 1]);
#pragma unroll
                        for (int c = 0; c < 4; c++)
                            *reinterpret_cast<uint4 *>(row_out + (cc * 4 + c) * chunk_stride) =
                                make_uint4(pk[4 * c], pk[4 * c + 1], pk[4 * c + 2], pk[4 * c + 3]);
                    }
                }
            }
            tc_fence_before();
            mbar_arrive(acc_empty);
            E12B_TR(2);
        }
        E12B_TR_DUMP("E2EP");
    }
    __syncwarp();
    tc_fence_before();
    __syncthreads();
    if (warp == 2) {
        tc_fence_after();
        tmem_dealloc(tmem_base, 512);
    }
}

#endif  // OTIF_E12B_BUILD

// ---------------------------------------------------------------------------
// E1 fused into E2, space-to-depth variant (e12s), with the resize fused in.  E1 (3x3,
// stride 2, 3 -> 32) is the stride-1 2x2 convolution over the space-to-depth image (one
// s2d pixel = the 2x2 proxy pixels (2Y + sy, 2X + sx) x 3 channels: 12 of 16 fp16
// channels (sy * 2 + sx) * 3 + c holding u - 128, exact), and for each of E2's four parity
// planes its four taps are LINEAR SHIFTS (0, -1, -pitch, -pitch - 1) within one of four
// s2d parity planes laid out with E2's plane pitch.  So E1's A operand is read straight
// from a staged halo ("slab") of the s2d planes through shifted descriptors — no per-row
// im2col gather (the critical role of the tile kernel, profiles/r02p_e12_source.md) — at
// 2.25x E1's MMA work (K = 4 taps x 16 instead of 32), which the tensor pipe has spare.
//
// The slab is built in shared memory by converter warps straight from the u8 source
// frames: with an even integer downscale FX x fy (every workload of SURVEY.md §8(d)) a
// proxy pixel is (sum of the 2x2 central source pixels + 2) >> 2 — exactly resize.cu's
// value — so stage 1 and E1's input conversion are one pass over the frames and the proxy
// image never exists in HBM (FX == 1: the input is the u8 proxy image itself).  Each CTA
// runs a contiguous range of tiles and the slab of tile t + 1 overlaps tile t's by
// 2 (pitch + 1) positions, which are copied on chip, so every s2d pixel is converted once.
//
// Roles (OTIF_E12S_THREADS = 640): warp 0 L2 prefetch of the next tile's source rows,
// warp 1 E1 MMA (KT x 4 per plane job), warp 2 TMEM allocator, warp 3 E2 MMA, warps 4-7 E1
// epilogue (ReLU, zero padding -> E2's A operand), 8-11 E2 epilogue, 12-19 converters.
// ---------------------------------------------------------------------------
#ifndef OTIF_E12S_THREADS
#define OTIF_E12S_THREADS 640   // 20 warps: 8 converter warps (with the L2 prefetch: C3 E1+E2 3.12 -> 2.87 ms, C2 -1%; 12 / 6 converter warps slower; profiles/r02y_e12s_threads_ab.log)
#endif
constexpr int kE12sThreads = OTIF_E12S_THREADS;
#ifndef OTIF_E12S_EPI1
#define OTIF_E12S_EPI1 4          // E1 epilogue warps (4 or 8); the rest after E2's 4 convert
#endif
constexpr int kE12sEpi1 = OTIF_E12S_EPI1 * 32;                  // E1 epilogue threads
constexpr int kE12sEpi2Warp = 4 + OTIF_E12S_EPI1;               // first E2 epilogue warp
constexpr int kE12sConvWarp = kE12sEpi2Warp + 4;                // first converter warp
constexpr int kE12sConv = kE12sThreads - kE12sConvWarp * 32;    // converter threads
// Channel slots of an s2d pixel (the s2d slot order): chunk A (K 0-7) = proxy row 2Y + 1: (sx 1,
// c 0-2), (sx 0, c 0-2), two bias slots; chunk B (K 8-15) = proxy row 2Y, same order, two
// zero slots.  The bias slots of every pixel inside the image hold 128.0 (fp16 0x5800):
// with tap (1, 1) weights (b_hi, b_lo) = E1's bias * 2^s split into two fp16 terms, the MMA
// adds E1's bias (x 2^(s+7), the accumulator scale) exactly as far as fp32 goes.  Taps
// (0, 0) and (0, 1) use only chunk A, so they share one K16 MMA (3 MMAs per E1 row, not 4).
constexpr uint32_t kE12sBiasCh = 0x58005800u;
#ifndef OTIF_E12S_PREFETCH
#define OTIF_E12S_PREFETCH 1      // tiles of source rows prefetched to L2 ahead of the converters (1: C2 E1+E2 1.156 -> 1.000 ms; 2: 1.081; profiles/r02y_e12s_prefetch_ab.log)
#endif
#ifndef OTIF_E12S_NOLOAD
#define OTIF_E12S_NOLOAD 0
#endif
constexpr int kE12sPrefetch = OTIF_E12S_PREFETCH;

struct E12sParams {
    const uint8_t *src;         // u8 NHWC frames [n, sh, sw, 3] (FX >= 2) or proxy image [n, hp, wp, 3] (FX == 1)
    int sh, sw, hp, wp, fy;
    int prefetch;               // source rows are 16-B aligned: L2 bulk prefetch usable
    int h1, w1, h2, w2, pitch;
    uint32_t fstride, mtot;
    FastDiv div_pitch, div_rpf, div_fstride;
    int PS;                     // slab positions per s2d plane = 256 + 2 (pitch + 1), rounded to 16
    int nslab;                  // slab buffers (1 or 2)
    int np;                     // plane buffers
    int ntiles;
    int group_ntaps[4], group_shift[4][9];
    const uint16_t *w1s;        // fp16 [4 taps][2 chunks][32 n][8] = w * 2^s (+ the bias terms, kE12sBiasCh)
    const uint16_t *wt2;        // as e12
    const float *b2;
    int out_kind;
    uint8_t *out;
    int64_t out_lcap;
    int out_c8, out_pitch;
    int64_t out_fstride;
};

// s2d parity plane and shift (positions) of E1 tap t = (ty, tx) for E2 plane g = (rp, cp)
__device__ __forceinline__ void e12s_tap(int g, int t, int pitch, int &h, int &shift) {
    const int rp = g >> 1, cp = g & 1, ty = t >> 1, tx = t & 1;
    h = (((rp + 1 + ty) & 1) << 1) | ((cp + 1 + tx) & 1);
    const int ry = (rp == 0 && ty == 0) ? -1 : 0, rx = (cp == 0 && tx == 0) ? -1 : 0;
    shift = ry * pitch + rx;
}

// bytes I and J of the little-endian byte string w[] as two zero-extended 16-bit lanes
template <int I, int J>
__device__ __forceinline__ uint32_t s2d_pair(const uint32_t *w) {
    if constexpr (I / 4 == J / 4) {
        return __byte_perm(w[I / 4], 0u, (I % 4) | (4 << 4) | ((J % 4) << 8) | (4 << 12));
    } else if constexpr (J / 4 == I / 4 + 1) {
        return __byte_perm(w[I / 4], w[J / 4], (I % 4) | ((J % 4 + 4) << 8)) & 0x00FF00FFu;
    } else {
        return __byte_perm(w[I / 4], 0u, (I % 4) | 0x4440) | __byte_perm(w[J / 4], 0u, 0x4044 | ((J % 4) << 8));
    }
}

// 16-bit lanes holding 0..255 -> fp16x2 of (v - 128), exact (0x6400 | v is 1024 + v)
__device__ __forceinline__ uint32_t s2d_f16(uint32_t v) { return sub_f16x2(0x64006400u | v, 0x64806480u); }
// 16-bit lanes holding sums of four bytes -> fp16x2 of ((s + 2) >> 2) - 128
__device__ __forceinline__ uint32_t s2d_avg_f16(uint32_t s) {
    return s2d_f16(((s + 0x00020002u) >> 2) & 0x00FF00FFu);
}

#ifndef OTIF_E12S_LD
#define OTIF_E12S_LD 0   // converter source loads: 0 ld.global.nc, 1 .cs, 2 ld.global, 3 .cg (L2 only)
#endif
template <typename T>
__device__ __forceinline__ T s2d_ld(const T *p) {
#if OTIF_E12S_LD == 1
    return __ldcs(p);
#elif OTIF_E12S_LD == 2
    return *p;
#elif OTIF_E12S_LD == 3
    return __ldcg(p);
#else
    return __ldg(p);
#endif
}

// Source bytes of two adjacent s2d columns X = 2xx, 2xx + 1 (proxy columns 4xx .. 4xx + 3)
// in one source row: w[] gets a little-endian byte string; O(xp, sx) is the offset of the
// first source pixel of proxy column 2X + sx (FX >= 2: the second one follows at + 3).
template <int FX> struct S2dRow;
template <> struct S2dRow<1> {      // proxy image: bytes 12xx .. 12xx + 11
    static constexpr int NW = 3;
    static constexpr int O(int xp, int sx) { return 6 * xp + 3 * sx; }
    __device__ __forceinline__ static void load(const uint8_t *row, int xx, uint32_t *w) {
        const uint32_t *s = reinterpret_cast<const uint32_t *>(row + 12 * xx);
        w[0] = s2d_ld(s); w[1] = s2d_ld(s + 1); w[2] = s2d_ld(s + 2);
    }
};
template <> struct S2dRow<2> {      // source columns 8xx .. 8xx + 7: bytes 24xx .. 24xx + 23
    static constexpr int NW = 6;
    static constexpr int O(int xp, int sx) { return 12 * xp + 6 * sx; }
    __device__ __forceinline__ static void load(const uint8_t *row, int xx, uint32_t *w) {
        const uint2 *s = reinterpret_cast<const uint2 *>(row + 24 * xx);
        const uint2 a = s2d_ld(s), b = s2d_ld(s + 1), c = s2d_ld(s + 2);
        w[0] = a.x; w[1] = a.y; w[2] = b.x; w[3] = b.y; w[4] = c.x; w[5] = c.y;
    }
};
template <> struct S2dRow<4> {      // source columns 16xx + {1, 2, 5, 6, 9, 10, 13, 14}: bytes 48xx + [0, 48)
    static constexpr int NW = 12;
    static constexpr int O(int xp, int sx) { return 24 * xp + 12 * sx + 3; }
    __device__ __forceinline__ static void load(const uint8_t *row, int xx, uint32_t *w) {
        const uint4 *s = reinterpret_cast<const uint4 *>(row + 48 * xx);
        const uint4 a = s2d_ld(s), b = s2d_ld(s + 1), c = s2d_ld(s + 2);
        w[0] = a.x; w[1] = a.y; w[2] = a.z; w[3] = a.w; w[4] = b.x; w[5] = b.y;
        w[6] = b.z; w[7] = b.w; w[8] = c.x; w[9] = c.y; w[10] = c.z; w[11] = c.w;
    }
};
template <> struct S2dRow<8> {      // source columns 32xx + {3, 4, 11, 12, 19, 20, 27, 28}: bytes 96xx + 8 + [0, 8), +24, +48, +72
    static constexpr int NW = 8;
    static constexpr int O(int xp, int sx) { return 16 * xp + 8 * sx + 1; }
    __device__ __forceinline__ static void load(const uint8_t *row, int xx, uint32_t *w) {
        const uint8_t *s = row + 96 * xx + 8;
#pragma unroll
        for (int k = 0; k < 4; k++) {
            const uint2 v = s2d_ld(reinterpret_cast<const uint2 *>(s + 24 * k));
            w[2 * k] = v.x; w[2 * k + 1] = v.y;
        }
    }
};

// one proxy pixel value (generic, byte loads): the right edge of odd proxy widths
template <int FX>
__device__ __forceinline__ uint32_t s2d_px_slow(const E12sParams &p, int f, int py, int px, int c) {
    if (py >= p.hp || px >= p.wp) return 128u;
    if (FX == 1) return __ldg(p.src + (((size_t)f * p.hp + py) * p.wp + px) * 3 + c);
    const int r0 = p.fy * py + p.fy / 2 - 1, c0 = FX * px + FX / 2 - 1;
    const uint8_t *a = p.src + (((size_t)f * p.sh + r0) * p.sw + c0) * 3 + c;
    const uint8_t *b = a + (size_t)p.sw * 3;
    return ((uint32_t)__ldg(a) + __ldg(a + 3) + __ldg(b) + __ldg(b + 3) + 2) >> 2;
}

// channel sums of one source row for s2d column parity XP into s0..s2 (16-bit lanes, the
// s2d slot order: (sx1 c0, sx1 c1), (sx1 c2, sx0 c0), (sx0 c1, sx0 c2))
template <int FX, int XP>
__device__ __forceinline__ void s2d_row_sums(const uint32_t *w, uint32_t &s0, uint32_t &s1, uint32_t &s2) {
    using R = S2dRow<FX>;
    constexpr int A = R::O(XP, 0), B = R::O(XP, 1);
    if constexpr (FX == 1) {
        s0 += s2d_pair<B, B + 1>(w);
        s1 += s2d_pair<B + 2, A>(w);
        s2 += s2d_pair<A + 1, A + 2>(w);
    } else {
        s0 += s2d_pair<B, B + 1>(w) + s2d_pair<B + 3, B + 4>(w);
        s1 += s2d_pair<B + 2, A>(w) + s2d_pair<B + 5, A + 3>(w);
        s2 += s2d_pair<A + 1, A + 2>(w) + s2d_pair<A + 4, A + 5>(w);
    }
}

// the 12 channels of s2d pixels (Y, 2xx) and (Y, 2xx + 1) of frame f as 6 fp16x2 words
// each, words 3 sy .. 3 sy + 2 = proxy row 2Y + sy in the s2d slot order; all source loads
// are issued before any is used (one memory latency per call)
template <int FX>
__device__ __forceinline__ void s2d_pixels(const E12sParams &p, int f, int Y, int xx, uint32_t (&o)[2][6]) {
    using R = S2dRow<FX>;
    if (4 * xx + 3 >= p.wp) {      // right edge of an odd proxy width: byte loads
#pragma unroll
        for (int xp = 0; xp < 2; xp++)
#pragma unroll
            for (int k = 0; k < 6; k++) {
                // slot s of proxy row sy: s < 3 -> (sx 1, c s), else (sx 0, c s - 3)
                const int sy = k / 3, s0 = 2 * (k % 3), s1 = s0 + 1, X = 2 * xx + xp;
                const uint32_t lo = s2d_px_slow<FX>(p, f, 2 * Y + sy, 2 * X + (s0 < 3), s0 % 3);
                const uint32_t hi = s2d_px_slow<FX>(p, f, 2 * Y + sy, 2 * X + (s1 < 3), s1 % 3);
                o[xp][k] = s2d_f16(lo | (hi << 16));
            }
        return;
    }
    const bool row1 = 2 * Y + 1 < p.hp;   // else the bottom edge of an odd proxy height
    constexpr int NR = FX == 1 ? 1 : 2;   // source rows per proxy row
    uint32_t w[2][NR][R::NW];
#pragma unroll
    for (int sy = 0; sy < 2; sy++) {
        const int py = 2 * Y + sy;
        const size_t r0 = FX == 1 ? (size_t)f * p.hp + py : (size_t)f * p.sh + p.fy * py + p.fy / 2 - 1;
        const uint8_t *row = p.src + r0 * (size_t)p.sw * 3;
#pragma unroll
        for (int d = 0; d < NR; d++) {
            if (sy == 0 || row1) {
                R::load(row + (size_t)d * p.sw * 3, xx, w[sy][d]);
            } else {
#pragma unroll
                for (int k = 0; k < R::NW; k++) w[sy][d][k] = 0u;
            }
        }
    }
#pragma unroll
    for (int sy = 0; sy < 2; sy++) {
        uint32_t a0 = 0, a1 = 0, a2 = 0, b0 = 0, b1 = 0, b2 = 0;
#pragma unroll
        for (int d = 0; d < NR; d++) {
            s2d_row_sums<FX, 0>(w[sy][d], a0, a1, a2);
            s2d_row_sums<FX, 1>(w[sy][d], b0, b1, b2);
        }
        if (FX == 1) {
            o[0][3 * sy] = s2d_f16(a0); o[0][3 * sy + 1] = s2d_f16(a1); o[0][3 * sy + 2] = s2d_f16(a2);
            o[1][3 * sy] = s2d_f16(b0); o[1][3 * sy + 1] = s2d_f16(b1); o[1][3 * sy + 2] = s2d_f16(b2);
        } else {
            o[0][3 * sy] = s2d_avg_f16(a0); o[0][3 * sy + 1] = s2d_avg_f16(a1); o[0][3 * sy + 2] = s2d_avg_f16(a2);
            o[1][3 * sy] = s2d_avg_f16(b0); o[1][3 * sy + 1] = s2d_avg_f16(b1); o[1][3 * sy + 2] = s2d_avg_f16(b2);
        }
        if (sy == 1 && !row1) {
#pragma unroll
            for (int k = 3; k < 6; k++) o[0][k] = o[1][k] = 0u;
        }
    }
}

// L2 prefetch of the source rows behind E2-layout rows [r0, r1) (row id = q / pitch)
template <int FX>
__device__ __forceinline__ void s2d_prefetch_rows(const E12sParams &p, int r0, int r1) {
    const size_t rb = (size_t)p.sw * 3;
    for (int rid = r0; rid < r1; rid++) {
        const int f = rid / (p.h2 + 1), gr = rid - f * (p.h2 + 1);
        if (gr == 0 || (uint32_t)f * p.fstride >= p.mtot) continue;   // top pad row / past the batch
        const int yy = gr - 1;
        if (FX == 1) {                 // proxy rows 4yy .. 4yy + 3 (as far as the image goes)
            const int py0 = 4 * yy, npy = min(4, p.hp - py0);
            if (npy > 0) bulk_prefetch_l2(p.src + ((size_t)f * p.hp + py0) * rb, (uint32_t)(npy * rb));
        } else {
            for (int py = 4 * yy; py < 4 * yy + 4 && py < p.hp; py++)
                bulk_prefetch_l2(p.src + ((size_t)f * p.sh + p.fy * py + p.fy / 2 - 1) * rb, (uint32_t)(2 * rb));
        }
    }
}

template <int KT, int FX>
__global__ void __launch_bounds__(kE12sThreads, 1) e12s_umma_kernel(const __grid_constant__ E12sParams p) {
    constexpr int kAccStages = 2, kE1Slots = 2;
    constexpr uint32_t kE1Col = kAccStages * 2 * 64;
    static_assert(kE1Col + kE1Slots * 32 * KT <= 512, "TMEM budget");
    extern __shared__ __align__(1024) uint8_t smem[];
    const int warp = threadIdx.x >> 5;
    const int lane = threadIdx.x & 31;
    constexpr int N2 = 64;
    constexpr int MT = 2;
    constexpr int P = 128 * KT;
    constexpr uint32_t kW2Bytes = 9 * 4 * N2 * 16;
    constexpr uint32_t kW1Bytes = 4 * 2 * 32 * 16;    // 4 taps x K16 x N32 fp16
    constexpr uint32_t kPlaneBytes = P * 64;
    const uint32_t slab_bytes = 8u * p.PS * 16;        // 4 planes x 2 chunks

    // the E1 MMAs of the last rows (P - 1 + pitch + 1 >= PS) read past a slab chunk into the
    // next one / the plane buffers: garbage for E1 rows that E2 never reads
    uint8_t *w2_s = smem;
    uint8_t *w1_s = w2_s + kW2Bytes;
    uint8_t *slab_s = w1_s + kW1Bytes;
    uint8_t *a2_s = slab_s + (size_t)p.nslab * slab_bytes;
    uint64_t *bars = reinterpret_cast<uint64_t *>(a2_s + (size_t)p.np * kPlaneBytes);
    uint64_t *slab_full = bars, *slab_empty = bars + 2;
    uint64_t *e1_full = bars + 4, *e1_empty = bars + 6;
    uint64_t *a2_full = bars + 8, *a2_empty = a2_full + kE12MaxPlaneBufs;
    uint64_t *acc_full = a2_empty + kE12MaxPlaneBufs, *acc_empty = acc_full + 2;
    uint32_t *tmem_slot = reinterpret_cast<uint32_t *>(acc_empty + 2);
    float *s_b2 = reinterpret_cast<float *>(tmem_slot + 4);

    // a contiguous range of tiles per CTA (consecutive slabs overlap)
    const int t_begin = (int)((int64_t)blockIdx.x * p.ntiles / gridDim.x);
    const int t_end = (int)((int64_t)(blockIdx.x + 1) * p.ntiles / gridDim.x);

    if (threadIdx.x == 0) {
        for (int i = 0; i < 2; i++) {
            mbar_init(&slab_full[i], kE12sConv); mbar_init(&slab_empty[i], 1);
            mbar_init(&acc_full[i], 1); mbar_init(&acc_empty[i], 128);
        }
        for (int i = 0; i < kE1Slots; i++) { mbar_init(&e1_full[i], 1); mbar_init(&e1_empty[i], kE12sEpi1); }
        for (int i = 0; i < kE12MaxPlaneBufs; i++) { mbar_init(&a2_full[i], kE12sEpi1); mbar_init(&a2_empty[i], 1); }
        fence_barrier_init();
    }
    if (warp == 2) tmem_alloc(tmem_slot, 512);
    for (uint32_t i = threadIdx.x; i < kW2Bytes / 16; i += blockDim.x)
        reinterpret_cast<uint4 *>(w2_s)[i] = reinterpret_cast<const uint4 *>(p.wt2)[i];
    for (uint32_t i = threadIdx.x; i < kW1Bytes / 16; i += blockDim.x)
        reinterpret_cast<uint4 *>(w1_s)[i] = reinterpret_cast<const uint4 *>(p.w1s)[i];
    if (threadIdx.x < N2) s_b2[threadIdx.x] = p.b2[threadIdx.x];
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem_base = *tmem_slot;

    if (warp >= kE12sConvWarp) {
        // ===== converters: slab positions j <-> E2-layout position q = q0 - pitch - 1 + j
        // of the 4 s2d parity planes, 2 chunks each; items (j, plane) with the plane's
        // column parity fastest, so lane pairs read adjacent source spans =====
        const int ct = threadIdx.x - (kE12sThreads - kE12sConv);
        const int PS = p.PS, nov = PS - 128 * MT;
        uint32_t sb = 0, sp = 0;
        for (int tile = t_begin; tile < t_end; tile++) {
            mbar_wait_sleep(&slab_empty[sb], sp ^ 1);
            uint8_t *slab = slab_s + (size_t)sb * slab_bytes;
            int j0 = 0;
            if (tile != t_begin && nov > 128 * MT) {
                // wide frames (overlap longer than a tile; two slabs): positions [256, nov) of
                // the previous slab were moved in, not converted, so after a converter-wide
                // barrier any thread moves any position
                const uint8_t *prev = slab_s + (size_t)(sb ^ 1) * slab_bytes;
                asm volatile("bar.sync 1, %0;" ::"n"(kE12sConv) : "memory");
#pragma unroll 1
                for (int ch = 0; ch < 8; ch++)
                    for (int j = ct; j < nov; j += kE12sConv)
                        *reinterpret_cast<uint4 *>(slab + ((size_t)ch * PS + j) * 16) =
                            *reinterpret_cast<const uint4 *>(prev + ((size_t)ch * PS + j + 128 * MT) * 16);
                j0 = nov;
            } else if (tile != t_begin) {
                // positions [256, PS) of the previous slab are [0, PS - 256) of this one: each
                // thread moves the ones it converted itself (no converter-wide barrier; with
                // one slab, in place: sources >= 256 > destinations, then one barrier before
                // the new positions [PS - 256, PS) overwrite sources)
                const uint8_t *prev = slab_s + (size_t)(p.nslab == 2 ? sb ^ 1 : sb) * slab_bytes;
                const int j0p = tile - 1 == t_begin ? 0 : nov;
#pragma unroll 1
                for (int it = ct; it < 2 * (PS - j0p); it += kE12sConv) {
                    const int j = j0p + ((it >> 5) << 4) + (it & 15), rh = (it >> 4) & 1;
                    if (j < 128 * MT) continue;
#pragma unroll
                    for (int c = 0; c < 4; c++) {
                        const size_t ch = 4 * rh + c;
                        *reinterpret_cast<uint4 *>(slab + (ch * PS + j - 128 * MT) * 16) =
                            *reinterpret_cast<const uint4 *>(prev + (ch * PS + j) * 16);
                    }
                }
                if (p.nslab == 1) asm volatile("bar.sync 1, %0;" ::"n"(kE12sConv) : "memory");
                j0 = nov;
            }
            const int q0 = tile * (128 * MT) - (p.pitch + 1);
            // items (j, s2d row parity rh), both column parities per item; half-warps run
            // 16 consecutive positions of one rh (adjacent source spans)
            const int items = 2 * (PS - j0);
#pragma unroll 1
            for (int it = ct; it < items; it += kE12sConv) {
                const int j = j0 + ((it >> 5) << 4) + (it & 15), rh = (it >> 4) & 1;
                const int q = q0 + j;
                uint32_t o[2][6] = {{0, 0, 0, 0, 0, 0}, {0, 0, 0, 0, 0, 0}};
                uint32_t bias[2] = {0u, 0u};    // channels 12, 13 of the pixels inside the image
                if (q >= 0 && (uint32_t)q < p.mtot) {
                    const uint32_t f = fdiv((uint32_t)q, p.div_fstride);
                    const uint32_t r = (uint32_t)q - f * p.fstride;
                    const uint32_t gr = fdiv(r, p.div_pitch);
                    const int yy = (int)gr - 1, xx = (int)(r - gr * (uint32_t)p.pitch) - 1;
                    const int Y = 2 * yy + rh;
                    if (yy >= 0 && xx >= 0 && Y < p.h1 && 2 * xx < p.w1) {
#if OTIF_E12S_NOLOAD == 1    // timing experiment only: no source loads (wrong results)
                        o[0][0] = (uint32_t)(Y + xx);
#elif OTIF_E12S_NOLOAD == 2  // timing experiment only: loads from a cache-resident corner
                        s2d_pixels<FX>(p, 0, Y & 7, xx & 15, o);
#else
                        s2d_pixels<FX>(p, (int)f, Y, xx, o);
#endif
                        bias[0] = kE12sBiasCh;
                        if (2 * xx + 1 < p.w1) {
                            bias[1] = kE12sBiasCh;
                        } else {
#pragma unroll
                            for (int k = 0; k < 6; k++) o[1][k] = 0u;
                        }
                    }
                }
#pragma unroll
                for (int xp = 0; xp < 2; xp++) {
                    const int h = 2 * rh + xp;
                    *reinterpret_cast<uint4 *>(slab + ((size_t)(2 * h) * PS + j) * 16) =
                        make_uint4(o[xp][3], o[xp][4], o[xp][5], bias[xp]);
                    *reinterpret_cast<uint4 *>(slab + ((size_t)(2 * h + 1) * PS + j) * 16) =
                        make_uint4(o[xp][0], o[xp][1], o[xp][2], 0u);
                }
            }
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
            mbar_arrive(&slab_full[sb]);
            if (++sb == (uint32_t)p.nslab) { sb = 0; sp ^= 1; }
        }
    } else if (warp == 0) {
        // ===== prefetcher: keeps the source rows of the tiles kE12sPrefetch ahead of the
        // converters on their way to L2 (their loads then wait for L2, not DRAM) =====
        if (lane == 0 && kE12sPrefetch > 0 && p.prefetch) {
            const uint32_t rows_q = (uint32_t)p.pitch;
            int pf_next = (int)(max(t_begin * (128 * MT) - (p.pitch + 1), 0) / rows_q);
            uint32_t sb = 0, sp = 0;
            for (int tile = t_begin; tile < t_end; tile++) {
                const int tl = min(tile + kE12sPrefetch, t_end - 1);
                const int pf_end = (int)(((uint32_t)(tl + 1) * (128 * MT) + p.pitch + 1) / rows_q) + 1;
                if (pf_end > pf_next) {
                    s2d_prefetch_rows<FX>(p, pf_next, pf_end);
                    pf_next = pf_end;
                }
                mbar_wait_sleep(&slab_full[sb], sp);     // the converters finished this tile
                if (++sb == (uint32_t)p.nslab) { sb = 0; sp ^= 1; }
            }
        }
    } else if (warp == 1) {
        // ===== E1 MMA issuer: per plane job KT sub-tiles x 4 shifted taps (K16 each) =====
        const uint32_t idesc1 = umma_idesc_f16(128, 32);
        const uint64_t w1d = umma_desc(smem_u32(w1_s), 512, 128);
        uint32_t J = 0, sb = 0, sp = 0;
        for (int tile = t_begin; tile < t_end; tile++) {
            mbar_wait(&slab_full[sb], sp);
            tc_fence_after();
            const uint32_t slab = smem_u32(slab_s + (size_t)sb * slab_bytes);
#pragma unroll 1
            for (int g = 0; g < 4; g++, J++) {
                mbar_wait(&e1_empty[J % kE1Slots], ((J / kE1Slots) & 1) ^ 1);
                tc_fence_after();
                const uint32_t d = tmem_base + kE1Col + (J % kE1Slots) * (32 * KT);
                // taps (0, 0) and (0, 1) read only chunk A: one K16 MMA takes both (its two
                // K halves LBO apart, in address order; weight block 0 or 1 to match);
                // taps (1, 0) and (1, 1) read chunks A and B of their plane (LBO = PS)
                int h0, s0, h1, s1;
                e12s_tap(g, 0, p.pitch, h0, s0);
                e12s_tap(g, 1, p.pitch, h1, s1);
                const uint32_t a00 = slab + (uint32_t)(2 * h0 * p.PS + (p.pitch + 1) + s0) * 16;
                const uint32_t a01 = slab + (uint32_t)(2 * h1 * p.PS + (p.pitch + 1) + s1) * 16;
                const bool fwd = a01 > a00;
                const uint64_t ad0 = umma_desc(fwd ? a00 : a01, fwd ? a01 - a00 : a00 - a01, 128);
                const uint64_t bd0 = w1d + ((fwd ? 0 : 1024) >> 4);
#pragma unroll
                for (int k = 0; k < KT; k++) umma_bf16_warp(d + k * 32, ad0 + ((k * 2048) >> 4), bd0, idesc1, 0u);
#pragma unroll 1
                for (int t = 2; t < 4; t++) {
                    int h, shift;
                    e12s_tap(g, t, p.pitch, h, shift);
                    const uint32_t a0 = slab + (uint32_t)(2 * h * p.PS + (p.pitch + 1) + shift) * 16;
                    const uint64_t ad = umma_desc(a0, p.PS * 16, 128);
                    const uint64_t bd = w1d + ((t * 1024) >> 4);
#pragma unroll
                    for (int k = 0; k < KT; k++) umma_bf16_warp(d + k * 32, ad + ((k * 2048) >> 4), bd, idesc1, 1u);
                }
                umma_commit_warp(&e1_full[J % kE1Slots]);
            }
            umma_commit_warp(&slab_empty[sb]);   // the slab is free once this tile's E1 MMAs read it
            if (++sb == (uint32_t)p.nslab) { sb = 0; sp ^= 1; }
        }
    } else if (warp == 3) {
        // ===== E2 MMA issuer (as e12) =====
        const uint32_t idesc2 = umma_idesc_bf16(128, N2);
        const uint64_t a2d = umma_desc(smem_u32(a2_s), P * 16, 128);
        const uint64_t w2d = umma_desc(smem_u32(w2_s), N2 * 16, 128);
        uint32_t pb = 0, pp = 0, acc = 0, accp = 0;
        for (int tile = t_begin; tile < t_end; tile++) {
            mbar_wait(&acc_empty[acc], accp ^ 1);
            tc_fence_after();
            const uint32_t d = tmem_base + acc * (MT * N2);
            int pos = 0;
            for (int g = 0; g < 4; g++) {
                mbar_wait(&a2_full[pb], pp);
                tc_fence_after();
                const uint64_t a = a2d + ((pb * kPlaneBytes) >> 4);
#pragma unroll 1
                for (int t = 0; t < p.group_ntaps[g]; t++, pos++) {
                    const uint64_t at = a + p.group_shift[g][t];
                    const uint64_t bt = w2d + ((pos * (4 * N2 * 16)) >> 4);
#pragma unroll
                    for (int s = 0; s < 2; s++)
#pragma unroll
                        for (int mm = 0; mm < MT; mm++)
                            umma_bf16_warp(d + mm * N2, at + ((2 * s * P * 16 + mm * 2048) >> 4), bt + ((2 * s * N2 * 16) >> 4),
                                           idesc2, (g == 0 && t == 0 && s == 0) ? 0u : 1u);
                }
                umma_commit_warp(&a2_empty[pb]);
                if (++pb == (uint32_t)p.np) { pb = 0; pp ^= 1; }
            }
            umma_commit_warp(&acc_full[acc]);
            if (++acc == kAccStages) { acc = 0; accp ^= 1; }
        }
    } else if (warp >= 4 && warp < kE12sEpi2Warp) {
        // ===== E1 epilogue (1 or 2 warpgroups, alternate sub-tiles): ReLU (the bias is in
        // the accumulator), zero padding, bf16 -> plane buffer (E2's A operand) =====
        constexpr int nwg = kE12sEpi1 / 128;
        const int wg = (warp - 4) >> 2;
        const int row = (threadIdx.x - 128) & 127;
        const int quarter = warp & 3;
        uint32_t J = 0, pb = 0, pp = 0;
        for (int tile = t_begin; tile < t_end; tile++) {
            const uint32_t q0 = (uint32_t)tile * (128 * MT);
            uint32_t vm[KT];
#pragma unroll
            for (int k = 0; k < KT; k++) {
                // which parity planes hold an E1 pixel at E2-layout position q (e12_decode)
                const uint32_t q = q0 + k * 128 + row;
                const uint32_t gr = fdiv(q, p.div_pitch);
                const int jc = (int)(q - gr * (uint32_t)p.pitch);
                const int i = (int)(gr - fdiv(gr, p.div_rpf) * (uint32_t)(p.h2 + 1));
                const bool in = q < p.mtot && i >= 1 && jc >= 1;
                const uint32_t r1 = 2 * i - 1 < p.h1, c1 = 2 * jc - 1 < p.w1;
                vm[k] = in ? (1u | (c1 << 1) | (r1 << 2) | ((r1 & c1) << 3)) : 0u;
            }
#pragma unroll 1
            for (int g = 0; g < 4; g++, J++) {
                mbar_wait(&a2_empty[pb], pp ^ 1);
                mbar_wait(&e1_full[J % kE1Slots], (J / kE1Slots) & 1);
                tc_fence_after();
                uint8_t *plane = a2_s + pb * kPlaneBytes;
                const uint32_t tacc = tmem_base + ((uint32_t)(quarter * 32) << 16) + kE1Col + (J % kE1Slots) * (32 * KT);
#pragma unroll 1
                for (int k = (int)(((uint32_t)wg + nwg * KT * 4 - J * KT % nwg) % nwg); k < KT; k += nwg) {
                    // E2 reads plane rows < 256 + pitch + 1: the rows of this warp's quarter
                    // past that (M = 128 granularity) are never read
                    if (k * 128 + quarter * 32 >= 128 * MT + p.pitch + 1) continue;
                    uint32_t vmk = vm[0];
#pragma unroll
                    for (int i = 1; i < KT; i++)
                        if (k == i) vmk = vm[i];
                    const bool valid = (vmk >> g) & 1;
                    uint32_t v[32];
                    tmem_ld32(tacc + k * 32, v);
                    uint32_t pk[16];
#pragma unroll
                    for (int j = 0; j < 16; j++)
                        pk[j] = valid ? pack_bf16x2_relu(__uint_as_float(v[2 * j]), __uint_as_float(v[2 * j + 1])) : 0u;
                    uint8_t *dst = plane + (size_t)(k * 128 + row) * 16;
#pragma unroll
                    for (int c = 0; c < 4; c++)
                        *reinterpret_cast<uint4 *>(dst + (size_t)c * P * 16) =
                            make_uint4(pk[4 * c], pk[4 * c + 1], pk[4 * c + 2], pk[4 * c + 3]);
                }
                tc_fence_before();
                mbar_arrive(&e1_empty[J % kE1Slots]);
                asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
                mbar_arrive(&a2_full[pb]);
                if (++pb == (uint32_t)p.np) { pb = 0; pp ^= 1; }
            }
        }
    } else if (warp >= kE12sEpi2Warp) {
        // ===== E2 epilogue (as e12) =====
        const int row = threadIdx.x - kE12sEpi2Warp * 32;
        const int quarter = warp & 3;
        uint32_t acc = 0, accp = 0;
        for (int tile = t_begin; tile < t_end; tile++) {
            mbar_wait_sleep(&acc_full[acc], accp);
            tc_fence_after();
#pragma unroll 1
            for (int mm = 0; mm < MT; mm++) {
                const uint32_t q = (uint32_t)tile * (128 * MT) + mm * 128 + row;
                const uint32_t f = fdiv(q, p.div_fstride);
                const uint32_t r = q - f * p.fstride;
                const uint32_t oy = fdiv(r, p.div_pitch);
                const int ox = (int)(r - oy * (uint32_t)p.pitch);
                const bool valid = q < p.mtot && (int)oy < p.h2 && ox < p.w2;
                int plane = 0;
                const int64_t L = layout_pixel(p.out_kind, p.out_pitch, p.out_fstride, (int)f, (int)oy, ox, plane);
                const uint32_t taddr = tmem_base + ((uint32_t)(quarter * 32) << 16) + acc * (MT * N2) + mm * N2;
                uint8_t *const row_out = p.out + ((int64_t)plane * p.out_c8 * p.out_lcap + L) * 16;
                const int64_t chunk_stride = p.out_lcap * 16;
#pragma unroll
                for (int cc = 0; cc < N2 / 32; cc++) {
                    uint32_t v[32];
                    tmem_ld32(taddr + cc * 32, v);
                    if (valid) {
                        uint32_t pk[16];
#pragma unroll
                        for (int j = 0; j < 16; j++)
                            pk[j] = pack_bf16x2_relu(__uint_as_float(v[2 * j]) + s_b2[cc * 32 + 2 * j],
                                                     __uint_as_float(v[2 * j + 1]) + s_b2[cc * 32 + 2 * j + 1]);
#pragma unroll
                        for (int c = 0; c < 4; c++)
                            *reinterpret_cast<uint4 *>(row_out + (cc * 4 + c) * chunk_stride) =
                                make_uint4(pk[4 * c], pk[4 * c + 1], pk[4 * c + 2], pk[4 * c + 3]);
                    }
                }
            }
            tc_fence_before();
            mbar_arrive(&acc_empty[acc]);
            if (++acc == kAccStages) { acc = 0; accp ^= 1; }
        }
    }
    __syncwarp();
    tc_fence_before();
    __syncthreads();
    if (warp == 2) {
        tc_fence_after();
        tmem_dealloc(tmem_base, 512);
    }
}

#define RC_PROXY(x)                     \
    do {                                \
        otif_status rc_ = (x);          \
        if (rc_ != OTIF_OK) return rc_; \
    } while (0)

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
    int kb, ncb, P, mt;
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
    // E1 fused into E2 (e12_umma_kernel); 0 = separate E1 kernel + E2 conv
    int e12;
    int e12_P, e12_np, e12_na1, e12_slab_rows, e12_slab_pitch;
    size_t e12_smem, e12_fixed, e12_unit;
    int e12_scale;                // s: E1 weights are scaled by 2^s (plan_e12)
    // space-to-depth variant of the fused E1+E2 kernel (e12s_umma_kernel)
    int e12s, e12s_PS, e12s_nslab, e12s_np;
    size_t e12s_smem;
    uint16_t *e12s_w1_dev;        // fp16 [4 taps][2 chunks][32][8] = bf16(w1) * 2^s
    // band variant of the fused E1+E2 kernel (e12b_umma_kernel); 0 = tile variant
    int e12b, e12b_R, e12b_PB, e12b_D, e12b_NR, e12b_RC, e12b_ring_pitch;
    size_t e12b_smem;
    uint16_t *e12_w1_dev;         // fp16 [4][32][8] = bf16(w1) * 2^s, K = kh*10 + kw*3 + c; bias parts at K = 9, 19, 29
    uint16_t *e12_w2_dev;         // E2's packed bf16 weights * 2^-(s+7)
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
        g.pitch = in_w + 1;     // one shared pad column per row (see the layout note)
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
    // (CTA pairs, cta_group::2 with M = 256, measured 1.3-1.7x slower than single CTAs here
    // because every stage hand-off is relayed through the peer's mbarrier:
    // profiles/r01_cta_pair.md; not built)
    g.P = (int)round_up(kTileM * g.mt + g.max_shift, 8);
}

static Layout input_layout(const GemmLayer &g, int n) {
    Layout l;
    l.kind = g.kind;
    l.planes = g.kind == 1 ? 1 : 4;
    l.pitch = g.pitch;
    l.fstride = g.fstride_unit;
    int64_t mtot = (int64_t)n * g.fstride_unit;
    l.lcap = round_up(round_up(mtot, (int64_t)kTileM * g.mt) + g.max_shift + 8, 16);
    l.c8 = g.cin / 8;
    l.bytes = (size_t)l.planes * l.c8 * l.lcap * 16;
    l.offset = 0;
    return l;
}

static size_t plan_workspace(const otif_proxy *p, int n, Layout lay[5]) {
    size_t off = 256;  // tag header
    for (int i = 0; i < 5; i++) {
        lay[i] = input_layout(p->L[i], n);
        if (i == 0 && p->e12 && (int64_t)n * p->L[0].fstride_unit + 4096 < (1ll << 31))
            lay[i].bytes = 0;   // E1 output stays on chip (fused kernel)
        lay[i].offset = off;
        off += round_up(lay[i].bytes, 256);
    }
    return off;
}

// fp16 bits of v if v is exactly representable in fp16
static bool f16_exact(float v, uint16_t *out) {
    const uint16_t sign = signbit(v) ? 0x8000 : 0;
    float a = fabsf(v);
    if (a == 0.0f) { *out = sign; return true; }
    if (!(a <= 65504.0f)) return false;
    if (a >= ldexpf(1.0f, -14)) {
        int ex;
        float m = frexpf(a, &ex);                 // a = m 2^ex, m in [0.5, 1)
        float frac = (m * 2.0f - 1.0f) * 1024.0f;  // a = (1 + frac/1024) 2^(ex-1)
        if (frac != floorf(frac)) return false;
        *out = (uint16_t)(sign | ((ex - 1 + 15) << 10) | (int)frac);
        return true;
    }
    float q = ldexpf(a, 24);
    if (q != floorf(q)) return false;
    *out = (uint16_t)(sign | (int)q);
    return true;
}

// Plan the fused E1+E2 kernel; returns false (separate kernels) when it does not apply.
// round to 11 significant bits (fp16's precision; the range is checked by f16_exact)
static float round_sig11(float x) {
    if (x == 0.0f) return 0.0f;
    int e;
    const float m = frexpf(x, &e);
    return ldexpf(rintf(ldexpf(m, 11)), e - 11);
}

// bf16 bits * 2^-k, if the result is an exact normal bf16 (or zero)
static bool bf16_scale_exact(uint16_t b, int k, uint16_t *out) {
    const int ex = (b >> 7) & 0xFF;
    if (ex == 0) {
        if (b & 0x7F) return false;
        *out = b;
        return true;
    }
    if (ex == 255 || ex - k < 1 || ex - k > 254) return false;
    *out = (uint16_t)((b & 0x807F) | ((ex - k) << 7));
    return true;
}

static void conv_smem(const GemmLayer &g, int &sa, int &sb, size_t &bytes);

// deepest (im2col stages, plane buffers) of the E1+E2 kernel within `budget` bytes
static bool e12_stages(size_t fixed, size_t unit, size_t budget, int &np, int &na1) {
    np = 0; na1 = 0;
    if (OTIF_E12_TS) {   // the im2col buffers live in TMEM: only plane buffers in shared memory
        for (int cand = kE12MaxPlaneBufs; cand >= 2 && !np; cand--)
            if (fixed + (size_t)cand * unit <= budget) { np = cand; na1 = 2; }
        return np != 0;
    }
    for (int cand_a1 = 2; cand_a1 >= 1 && !np; cand_a1--)
        for (int cand = kE12MaxPlaneBufs; cand >= 2 && !np; cand--)
            if (fixed + (size_t)(cand_a1 + cand) * unit <= budget) { np = cand; na1 = cand_a1; }
    return np != 0;
}

static bool plan_e12(otif_proxy *p, const float *w1 /* [32][3][3][3] */, const float *b1 /* [32] */) {
    const GemmLayer &g = p->L[0];
    if (p->d.n_strided < 2 || g.kind != 2 || g.cin != 32 || g.cout != 64) return false;
    float maxabs = 0.0f;
    for (int i = 0; i < 32 * 27; i++) maxabs = fmaxf(maxabs, fabsf(bf16_to_f32(f32_to_bf16_rne(w1[i]))));
    int s = 0;
    if (maxabs > 0.0f) {
        int ex;
        frexpf(32768.0f / maxabs, &ex);           // 2^(ex-1) <= 32768/maxabs < 2^ex
        s = ex - 1;
    }
    if (s < -20 || s > 40) return false;
    std::vector<uint16_t> wh(4 * 32 * 8, 0);
    for (int o = 0; o < 32; o++)
        for (int k = 0; k < 32; k++) {
            const int kh = k / 10, slot = k % 10;
            if (kh > 2 || slot > 8) continue;
            const int kw = slot / 3, c = slot % 3;
            const float v = ldexpf(bf16_to_f32(f32_to_bf16_rne(w1[((o * 3 + kh) * 3 + kw) * 3 + c])), s);
            uint16_t h;
            if (!f16_exact(v, &h)) return false;
            wh[((k / 8) * 32 + o) * 8 + (k % 8)] = h;
        }
    // the bias rides in the MMA: A holds 128 at K = 9, 19, 29 (slot 9 of each kernel row),
    // B holds b * 2^s split exactly into three fp16 parts, so acc = 2^(s+7) (sum + b)
    for (int o = 0; o < 32; o++) {
        const float x = ldexpf(b1[o], s);
        if (ldexpf(x, -s) != b1[o]) return false;
        const float hi = round_sig11(x), r = x - hi, mid = round_sig11(r), lo = r - mid;
        const float parts[3] = {hi, mid, lo};
        for (int kh = 0; kh < 3; kh++) {
            uint16_t h;
            if (!f16_exact(parts[kh], &h)) return false;
            const int k = kh * 10 + 9;
            wh[((k / 8) * 32 + o) * 8 + (k % 8)] = h;
        }
    }
    // E2 reads E1's activations scaled by 2^(s+7): scale its weights by 2^-(s+7) (exact)
    std::vector<uint16_t> w2((size_t)9 * 4 * 64 * 8);
    if (cudaMemcpy(w2.data(), g.wpk_dev, w2.size() * 2, cudaMemcpyDeviceToHost) != cudaSuccess) return false;
    for (auto &b : w2)
        if (!bf16_scale_exact(b, s + 7, &b)) return false;
    const int pitch = g.pitch;
    const int P = (int)round_up(256 + pitch + 1, 128);
    if (P / 128 < 3 || P / 128 > 4) return false;      // e12_umma_kernel<KT> instances
    const int npr = (P - 1) / pitch + 2;
    const int slab_rows = 4 * npr + 1;
    const int slab_pitch = (int)round_up(16 + 3 * p->d.in_w + 32, 16);
    const size_t fixed = 9 * 4 * 64 * 16 + 4 * 32 * 16 + 2 * (size_t)slab_rows * slab_pitch + 64 * 8 + 16 + 96 * 4 + 1024;
    const size_t a1 = (size_t)P * 64, plane = (size_t)P * 64;
    int np = 0, na1 = 0;
    if (!e12_stages(fixed, a1, 227 * 1024, np, na1)) return false;
    if (cudaMalloc(&p->e12_w1_dev, wh.size() * 2) != cudaSuccess) return false;
    cudaMemcpy(p->e12_w1_dev, wh.data(), wh.size() * 2, cudaMemcpyHostToDevice);
    if (cudaMalloc(&p->e12_w2_dev, w2.size() * 2) != cudaSuccess) return false;
    cudaMemcpy(p->e12_w2_dev, w2.data(), w2.size() * 2, cudaMemcpyHostToDevice);
    p->e12_P = P;
    p->e12_np = np;
    p->e12_slab_rows = slab_rows;
    p->e12_slab_pitch = slab_pitch;
    p->e12_na1 = na1;
    p->e12_smem = fixed + (OTIF_E12_TS ? 0 : (size_t)na1 * a1) + (size_t)np * plane;
    p->e12_fixed = fixed;
    p->e12_unit = a1;
    p->e12_scale = s;
    return true;
}

#ifndef OTIF_E12S
#define OTIF_E12S 1   // space-to-depth variant of the fused E1+E2 kernel where it applies (A/B: 0 = tile)
#endif
// Plan the s2d variant (needs plan_e12's scale s and scaled E2 weights): E1's weights as
// four 2x2-tap K16 blocks over the s2d channels (sy * 2 + sx) * 3 + c, bias * 2^(s+7).
static bool plan_e12s(otif_proxy *p, const float *w1 /* [32][3][3][3] */, const float *b1) {
    if (!OTIF_E12S || !p->e12) return false;
    const GemmLayer &g = p->L[0];
    const int KT = p->e12_P / 128;
    const int pitch = g.pitch;
    const int PS = (int)round_up(128 * 2 + 2 * (pitch + 1), 16);
    const int s = p->e12_scale;
    // s2d channel slots (the s2d slot order): chunk A = (sy 1: sx 1 c0-2, sx 0 c0-2, bias, bias),
    // chunk B = (sy 0: sx 1 c0-2, sx 0 c0-2, 0, 0).  Weight blocks [K half][32 n][8]:
    // 0 = (tap (0,0) A | tap (0,1) A), 1 = (tap (0,1) A | tap (0,0) A),
    // 2 = (tap (1,0) A | tap (1,0) B), 3 = (tap (1,1) A | tap (1,1) B)
    std::vector<uint16_t> w((size_t)4 * 2 * 32 * 8, 0);
    auto put = [&](int blk, int half, int t, int chunk) -> bool {
        const int ty = t >> 1, tx = t & 1, sy = chunk == 0 ? 1 : 0;
        for (int o = 0; o < 32; o++)
            for (int slot = 0; slot < 6; slot++) {
                const int sx = slot < 3 ? 1 : 0, c = slot % 3;
                // tap (ty, tx) reads s2d row y - 1 + ty: image row 2(y - 1 + ty) + sy = 2y - 1 + kh
                const int kh = 2 * ty + sy - 1, kw = 2 * tx + sx - 1;
                if (kh < 0 || kh > 2 || kw < 0 || kw > 2) continue;
                const float v = ldexpf(bf16_to_f32(f32_to_bf16_rne(w1[((o * 3 + kh) * 3 + kw) * 3 + c])), s);
                uint16_t h;
                if (!f16_exact(v, &h)) return false;
                w[(((size_t)blk * 2 + half) * 32 + o) * 8 + slot] = h;
            }
        return true;
    };
    if (!(put(0, 0, 0, 0) && put(0, 1, 1, 0) && put(1, 0, 1, 0) && put(1, 1, 0, 0) && put(2, 0, 2, 0) &&
          put(2, 1, 2, 1) && put(3, 0, 3, 0) && put(3, 1, 3, 1)))
        return false;
    // E1's bias on chunk A slots 6, 7 (128.0 inside the image) of tap (1, 1):
    // b * 2^s = hi + lo in two fp16 terms (hi * 128 + lo * 128 is exact in the fp32 accumulator)
    for (int o = 0; o < 32; o++) {
        const float v = ldexpf(b1[o], s);
        const __half hi = __float2half_rn(v);
        const __half lo = __float2half_rn(v - __half2float(hi));
        if (!isfinite(__half2float(hi))) return false;
        w[(((size_t)3 * 2 + 0) * 32 + o) * 8 + 6] = __half_as_ushort(hi);
        w[(((size_t)3 * 2 + 0) * 32 + o) * 8 + 7] = __half_as_ushort(lo);
    }
    // weights, then (after the slabs and plane buffers) the barriers, TMEM slot and E2 bias
    // (432 B, 1 KB reserved); the 1 KB static reservation of the kernel's aligned buffer is
    // added in the fit test below
    const size_t fixed = 9 * 4 * 64 * 16 + 4 * 2 * 32 * 16 + 1024;
    const size_t slab = (size_t)8 * PS * 16, plane = (size_t)p->e12_P * 64;
    int nslab = 0, np = 0;
#ifndef OTIF_E12S_NSLAB
#define OTIF_E12S_NSLAB 2
#endif
#ifndef OTIF_E12S_NP
#define OTIF_E12S_NP 2      // max plane buffers (3 measured slower: 1.33 vs 1.18 ms, less L1 for the converters)
#endif
    // Plane buffers: two (the E1 epilogue writes one while E2 reads the other) where they
    // fit, else one (the 640-wide C4d).  Before the L2 prefetch of the source rows, one
    // plane buffer paid on wide frames because it left more L1 to the converters' DRAM
    // loads (C3 3.71 -> 3.35 ms, profiles/r02y_e12s_smem_ab.log); with the prefetch their
    // loads hit L2 and two buffers are faster again (C4b 0.236 -> 0.213 ms, C3 3.23 -> 3.17,
    // profiles/r02y_e12s_carve_ab.log).
    for (int cs = OTIF_E12S_NSLAB; cs >= 1 && !np; cs--)
        for (int cp = OTIF_E12S_NP; cp >= 1 && !np; cp--)
            if (fixed + cs * slab + cp * plane + 1024 /* static */ <= 227 * 1024) { nslab = cs; np = cp; }
    // an overlap longer than a tile (proxy width > 508) is moved between two slabs
    if (!np || KT < 3 || KT > 4 || (PS - 256 > 256 && nslab < 2)) return false;
    if (cudaMalloc(&p->e12s_w1_dev, w.size() * 2) != cudaSuccess) return false;
    cudaMemcpy(p->e12s_w1_dev, w.data(), w.size() * 2, cudaMemcpyHostToDevice);
    p->e12s_PS = PS; p->e12s_nslab = nslab; p->e12s_np = np;
    p->e12s_smem = fixed + nslab * slab + np * plane;
    return true;
}

// Plan the band variant (needs the tile variant's scaled weights): R E2 rows per band with
// R * pitch <= 256, plane buffers of PB >= 256 + pitch + 1 rows; fits TMEM (128 + PB
// columns) and shared memory.
static bool plan_e12b(otif_proxy *p) {
    if (!OTIF_E12B || !p->e12) return false;
    const GemmLayer &g = p->L[0];
    const int pitch = g.pitch;
    const int R = 256 / pitch;
    if (R < 1) return false;
    const int PB = (int)round_up(256 + pitch + 1, 32);
    if (128 + PB > 512) return false;
    const int D = (PB - 1) / pitch;
    const int NR = 4 * D + 5;
    const int RC = 2 * NR;
    const int ring_pitch = (int)round_up(16 + 3 * p->d.in_w + 32, 16);
    const size_t smem = (size_t)(4 * PB / 128) * 8192 + (size_t)4 * PB * 64 + 3 * 4096 + 2048 +
                        (size_t)RC * ring_pitch + 32 * 8 + 16 + 64 * 4 + 1024;
    if (smem > 227 * 1024) return false;
    p->e12b_R = R; p->e12b_PB = PB; p->e12b_D = D; p->e12b_NR = NR; p->e12b_RC = RC;
    p->e12b_ring_pitch = ring_pitch;
    p->e12b_smem = smem;
    return true;
}

// kernel launches of one launch_proxy call (workspace zero + tag, E1+E2 fused or E1 and E2, E3..D1)
int proxy_launches(const otif_proxy *p) { return p->e12 ? 7 : 8; }

static void conv_smem(const GemmLayer &g, int &sa, int &sb, size_t &bytes) {
    size_t a = (size_t)(g.kb / 8) * g.P * 16;
    size_t b = (size_t)g.cout * g.kb * 2;
    size_t fixed = (3 * kMaxStagesA + 3 * kMaxStagesB + 4) * 8 + 16 + 2 * 256 * 4 + 4 * 256 * 4 + 1024;
    const size_t budget = 220 * 1024;
    sa = 2; sb = 2;
    // grow B (weights stream every tap) first, then A (deeper rings measured no faster,
    // DESIGN.md §11)
    const int sb_max = 6;
    while (sb < kMaxStagesB && sa * a + (sb + 1) * b + fixed <= budget && sb < sb_max) sb++;
    while (sa < kMaxStagesA && (sa + 1) * a + sb * b + fixed <= budget && sa < 3) sa++;
    bytes = sa * a + sb * b + fixed;
}

// Lay the workspace out for the largest batch it can hold (so every batch size up to it
// shares one layout and one zero-initialisation: a smaller final batch does not re-zero)
// and enqueue the one-time zeroing (a no-op while the header tag matches).
static otif_status prepare_ws(const otif_proxy *p, int n, uint8_t *ws, size_t ws_bytes, cudaStream_t stream,
                              Layout lay[5]) {
    size_t need = plan_workspace(p, n, lay);
    if (ws_bytes < need) {
        set_error("otif_proxy_score: workspace %zu B < required %zu B", ws_bytes, need);
        return OTIF_ENOMEM;
    }
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
    return OTIF_OK;
}

// Source of the s2d variant's converters: FX = 1 (the u8 proxy image) or the frames with
// an even integer downscale FX x fy, FX in {2, 4, 8} (0: the s2d variant does not apply).
static int e12s_fx(const otif_proxy *p, int n, const uint8_t *src, int sh, int sw, int *fy) {
    if (!p->e12s || n <= 0 || !(p->e12 && (int64_t)n * p->L[0].fstride_unit + 4096 < (1ll << 31))) return 0;
    const int hp = p->d.in_h, wp = p->d.in_w;
    if (sh == hp && sw == wp) {
        *fy = 1;
        return ((uintptr_t)src & 3) == 0 && (wp * 3) % 4 == 0 ? 1 : 0;
    }
    if (sw % wp || sh % hp) return 0;
    const int fx = sw / wp;
    *fy = sh / hp;
    if (!(fx == 2 || fx == 4 || fx == 8) || *fy < 2 || *fy % 2) return 0;
    return ((uintptr_t)src & 15) == 0 && (sw * 3) % 16 == 0 ? fx : 0;
}

// The pipeline skips stage 1 when the proxy reads its frames directly (e12s_umma_kernel).
bool proxy_fuses_resize(const otif_proxy *p, int n, const uint8_t *src, int sh, int sw) {
    int fy;
    return e12s_fx(p, n, src, sh, sw, &fy) >= 2;
}

// evs (optional): 6 events recorded after E1 (prep) and after each of the 5 GEMM layers;
// frames (optional, proxy_fuses_resize true): the source frames [n, sh, sw, 3], read by
// the fused E1+E2 kernel in place of the proxy image (img unused)
otif_status launch_proxy(const otif_proxy *p, const uint8_t *img, int n, float *scores, uint8_t *ws,
                         size_t ws_bytes, cudaStream_t stream, cudaEvent_t *evs, PackJob *pj,
                         const uint8_t *frames, int sh, int sw, unsigned long long *pj_snap) {
    Layout lay[5];
    otif_status pst = prepare_ws(p, n, ws, ws_bytes, stream, lay);
    if (pst != OTIF_OK) return pst;

    const bool e12 = p->e12 && (int64_t)n * p->L[0].fstride_unit + 4096 < (1ll << 31);
#if OTIF_E12B_BUILD
    if (e12 && p->e12b) {
        // E1 fused into E2, band variant: one kernel writes E3's input
        if (evs) OTIF_CUDA(cudaEventRecord(evs[0], stream));
        const GemmLayer &g = p->L[0];
        E12bParams e;
        memset(&e, 0, sizeof(e));
        e.img = img; e.n = n; e.hp = p->d.in_h; e.wp = p->d.in_w; e.row_bytes = 3 * p->d.in_w;
        e.h1 = p->e1_oh; e.w1 = p->e1_ow; e.h2 = g.out_h; e.w2 = g.out_w; e.pitch = g.pitch;
        e.R = p->e12b_R;
        e.nbpf = (e.h2 + e.R - 1) / e.R;
        e.njobs = n * e.nbpf;
        e.PB = p->e12b_PB; e.D = p->e12b_D; e.NR = p->e12b_NR; e.RC = p->e12b_RC;
        e.ring_pitch = p->e12b_ring_pitch;
        e.bulk = (e.row_bytes % 16 == 0) && (((uintptr_t)img & 15) == 0);
        e.div_pitch = make_fastdiv((uint32_t)g.pitch);
        e.div_PB = make_fastdiv((uint32_t)e.PB);
        e.div_RC = make_fastdiv((uint32_t)e.RC);
        e.wt1 = p->e12_w1_dev; e.wt2 = p->e12_w2_dev; e.b2 = g.bias_dev;
        for (int i = 0; i < 4; i++) {
            e.group_ntaps[i] = g.group_ntaps[i];
            for (int t = 0; t < 9; t++) e.group_shift[i][t] = g.group_shift[i][t];
        }
        e.out_kind = lay[1].kind; e.out = ws + lay[1].offset; e.out_lcap = lay[1].lcap;
        e.out_c8 = lay[1].c8; e.out_pitch = lay[1].pitch; e.out_fstride = lay[1].fstride;
        OTIF_CUDA(cudaFuncSetAttribute(e12b_umma_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                       (int)p->e12b_smem));
        const int grid = e.njobs < p->num_sms ? e.njobs : p->num_sms;
        e12b_umma_kernel<<<grid, kE12bThreads, p->e12b_smem, stream>>>(e);
        OTIF_LAUNCH_CHECK();
        if (evs) OTIF_CUDA(cudaEventRecord(evs[1], stream));
    } else
#endif
    int s_fy = 1;
    const int s_fx = frames ? e12s_fx(p, n, frames, sh, sw, &s_fy) : e12s_fx(p, n, img, p->d.in_h, p->d.in_w, &s_fy);
    if (frames && s_fx < 2) {
        set_error("launch_proxy: frames %dx%d are not an even downscale read by the fused kernel", sw, sh);
        return OTIF_EINVAL;
    }
    if (e12 && s_fx) {
        // E1 fused into E2, s2d variant, reading the frames (or the proxy image) directly
        if (evs) OTIF_CUDA(cudaEventRecord(evs[0], stream));
        const GemmLayer &g = p->L[0];
        E12sParams e;
        memset(&e, 0, sizeof(e));
        e.src = frames ? frames : img;
        e.sh = frames ? sh : p->d.in_h; e.sw = frames ? sw : p->d.in_w;
        e.hp = p->d.in_h; e.wp = p->d.in_w; e.fy = s_fy;
        e.prefetch = kE12sPrefetch > 0 && ((uintptr_t)e.src & 15) == 0 && ((size_t)e.sw * 3) % 16 == 0;
        e.h1 = p->e1_oh; e.w1 = p->e1_ow; e.h2 = g.out_h; e.w2 = g.out_w; e.pitch = g.pitch;
        e.fstride = (uint32_t)g.fstride_unit; e.mtot = (uint32_t)((int64_t)n * g.fstride_unit);
        e.div_pitch = make_fastdiv((uint32_t)g.pitch);
        e.div_rpf = make_fastdiv((uint32_t)g.out_h + 1);
        e.div_fstride = make_fastdiv((uint32_t)g.fstride_unit);
        e.PS = p->e12s_PS; e.nslab = p->e12s_nslab; e.np = p->e12s_np;
        e.ntiles = (int)cdiv(e.mtot, 256);
        for (int i = 0; i < 4; i++) {
            e.group_ntaps[i] = g.group_ntaps[i];
            for (int t = 0; t < 9; t++) e.group_shift[i][t] = g.group_shift[i][t];
        }
        e.w1s = p->e12s_w1_dev;
        e.wt2 = p->e12_w2_dev; e.b2 = g.bias_dev;
        e.out_kind = lay[1].kind; e.out = ws + lay[1].offset; e.out_lcap = lay[1].lcap;
        e.out_c8 = lay[1].c8; e.out_pitch = lay[1].pitch; e.out_fstride = lay[1].fstride;
        void (*kern)(E12sParams) = nullptr;
        const bool k3 = p->e12_P == 384;
        switch (s_fx) {
            case 1: kern = k3 ? e12s_umma_kernel<3, 1> : e12s_umma_kernel<4, 1>; break;
            case 2: kern = k3 ? e12s_umma_kernel<3, 2> : e12s_umma_kernel<4, 2>; break;
            case 4: kern = k3 ? e12s_umma_kernel<3, 4> : e12s_umma_kernel<4, 4>; break;
            default: kern = k3 ? e12s_umma_kernel<3, 8> : e12s_umma_kernel<4, 8>; break;
        }
        OTIF_CUDA(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)p->e12s_smem));
        const int grid = e.ntiles < p->num_sms ? e.ntiles : p->num_sms;
        kern<<<grid, kE12sThreads, p->e12s_smem, stream>>>(e);
        OTIF_LAUNCH_CHECK();
        if (evs) OTIF_CUDA(cudaEventRecord(evs[1], stream));
    } else if (e12) {
        // E1 fused into E2: one kernel writes E3's input
        if (evs) OTIF_CUDA(cudaEventRecord(evs[0], stream));
        const GemmLayer &g = p->L[0];
        E12Params e;
        memset(&e, 0, sizeof(e));
        e.img = img; e.n = n; e.hp = p->d.in_h; e.wp = p->d.in_w; e.row_bytes = 3 * p->d.in_w;
        e.h1 = p->e1_oh; e.w1 = p->e1_ow;
        e.h2 = g.out_h; e.w2 = g.out_w; e.pitch = g.pitch;
        e.fstride = (uint32_t)g.fstride_unit; e.mtot = (uint32_t)((int64_t)n * g.fstride_unit);
        e.div_pitch = make_fastdiv((uint32_t)g.pitch);
        e.div_rpf = make_fastdiv((uint32_t)g.out_h + 1);
        e.div_fstride = make_fastdiv((uint32_t)g.fstride_unit);
        e.P = p->e12_P; e.np = p->e12_np; e.na1 = p->e12_na1;
        e.ntiles = (int)cdiv(e.mtot, 256);
        e.slab_rows = p->e12_slab_rows; e.slab_pitch = p->e12_slab_pitch;
        e.bulk = (e.row_bytes % 16 == 0) && (((uintptr_t)img & 15) == 0);
#ifdef OTIF_E12_TRACE_BUILD
        if (const char *x = getenv("OTIF_E12_TRACE")) e.trace = atoi(x);
#endif
        for (int i = 0; i < 4; i++) {
            e.group_ntaps[i] = g.group_ntaps[i];
            for (int t = 0; t < 9; t++) e.group_shift[i][t] = g.group_shift[i][t];
        }
        e.wt1 = p->e12_w1_dev;
        e.wt2 = p->e12_w2_dev; e.b2 = g.bias_dev;
        e.out_kind = lay[1].kind; e.out = ws + lay[1].offset; e.out_lcap = lay[1].lcap;
        e.out_c8 = lay[1].c8; e.out_pitch = lay[1].pitch; e.out_fstride = lay[1].fstride;
        e.pj = OTIF_PJ_E12 > 0 ? pj : nullptr;
        auto kern = e.P == 384 ? e12_umma_kernel<3> : e12_umma_kernel<4>;
        OTIF_CUDA(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)p->e12_smem));
        const int grid = e.ntiles < p->num_sms ? e.ntiles : p->num_sms;
        kern<<<grid, kE12Threads, p->e12_smem, stream>>>(e);
        OTIF_LAUNCH_CHECK();
        if (evs) OTIF_CUDA(cudaEventRecord(evs[1], stream));
    }
    // E1
    if (!e12) {
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
    for (int li = e12 ? 1 : 0; li < 5; li++) {
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
        // fused copy warps only in the tensor-bound layers past E3 (E3 is HBM-bound)
        c.pj = ((OTIF_PJ_LAYERS >> li) & 1) ? pj : nullptr;
        c.mtot = (int64_t)n * g.fstride_unit;
        c.ntiles = (int)cdiv(c.mtot, (int64_t)kTileM * g.mt);
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
        // head layer with N = 128: swapped operands (see conv_umma_kernel)
        const bool swap = c.out_kind == 3 && g.mt == 2 && g.cout == 128;
        // weight-sharing CTA pairs (CL = 2) for the layers in OTIF_CONV_CL_LAYERS
#if OTIF_CONV_CL_LAYERS
        const bool pair = ((OTIF_CONV_CL_LAYERS >> li) & 1) && c.ntiles >= 2 && p->num_sms >= 2;
#else
        constexpr bool pair = false;
#endif
        if (pair) {
#if OTIF_CONV_CL_LAYERS
            const int pairs_max = p->num_sms / 2;
            const int ntp = (c.ntiles + 1) / 2;
            const int pairs = ntp < pairs_max ? ntp : pairs_max;
            auto kern = swap ? conv_umma_kernel<2, true, 2>
                             : (g.mt == 4 ? conv_umma_kernel<4, false, 2>
                                          : (g.mt == 2 ? conv_umma_kernel<2, false, 2> : conv_umma_kernel<1, false, 2>));
            OTIF_CUDA(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
            cudaLaunchConfig_t cfg = {};
            cfg.gridDim = dim3(2 * pairs);
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
#endif
        } else {
            int grid = c.ntiles < p->num_sms ? c.ntiles : p->num_sms;
            if (grid < 1) grid = 1;
            auto kern = swap ? conv_umma_kernel<2, true>
                             : (g.mt == 4 ? conv_umma_kernel<4> : (g.mt == 2 ? conv_umma_kernel<2> : conv_umma_kernel<1>));
            OTIF_CUDA(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
            kern<<<grid, kConvThreads, smem, stream>>>(c);
        }
        OTIF_LAUNCH_CHECK();
        if (evs) OTIF_CUDA(cudaEventRecord(evs[1 + li], stream));
        // timing only: the pack-unit claim counter after this layer (which layer carried how
        // much of the fused copy)
        if (pj && pj_snap) OTIF_CUDA(cudaMemcpyAsync(pj_snap + li, &pj->next, 8, cudaMemcpyDeviceToDevice, stream));
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
                                pk[((((size_t)cb * 9 + pos) * chunks + j) * g.cout + nn) * 8 + e] = f32_to_bf16_rne(v);
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
    if (rc == OTIF_OK) p->e12 = plan_e12(p, weights + offs[0], weights + offs[0] + 32 * 27) ? 1 : 0;
    if (rc == OTIF_OK) p->e12b = plan_e12b(p) ? 1 : 0;
    if (rc == OTIF_OK && !p->e12b) p->e12s = plan_e12s(p, weights + offs[0], weights + offs[0] + 32 * 27) ? 1 : 0;
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
    mix(p->e12);
    mix(p->e12b);
    mix(p->e12s);
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
    if (p->e12_w1_dev) cudaFree(p->e12_w1_dev);
    if (p->e12_w2_dev) cudaFree(p->e12_w2_dev);
    if (p->e12s_w1_dev) cudaFree(p->e12s_w1_dev);
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
    return launch_proxy(p, img, n, scores, (uint8_t *)workspace, ws_bytes, stream, nullptr, nullptr, nullptr, 0, 0, nullptr);
}
