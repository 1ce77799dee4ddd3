// train.cu — §8(f) NEXT-3, proxy training labels and training on sm_100a.
//
//   labels_kernel    P:L139 label 1 at every cell a detection intersects (thread per box).
//   tc_gemm_kernel<Op, BN> the tcgen05 implicit GEMM (3xTF32 split, fp32 accumulation in
//                    TMEM, 128 x BN tiles, gathers through the Op) — the default; and
//   sgemm_kernel<Op> the fp32 SIMT version of the same template (64 x 64 x 16 tiles, 4 x 4 per
//                    thread, OTIF_TRAIN_SIMT=1), instantiated for the three convolution products:
//                      FwdOp    y = ReLU(conv(x, W) + b)           M = pixels, N = Cout, K = 9 Cin
//                      DgradOp  dx = conv^T(dy, W) ⊙ [x > 0]        M = input pixels, N = Cin, K = 9 Cout
//                      WgradOp  dW | db = dy^T · im2col(x) | Σ dy   M = Cout, N = 9 Cin + 1, K = pixels
//                    (split-K partials for WgradOp, reduced in a fixed order: deterministic).
//   head_kernel      D2 (1x1, dec -> 1) + sigmoid + mean BCE (reading R26) + ∂/∂z, the D1
//                    pre-activation gradient and per-warp D2 weight-gradient partials.
//   adam_kernel      reading R27, fp32 master weights.
//
// Training runs in fp32 (weights, activations, gradients; the 3xTF32 products keep fp32
// accuracy, so the gradients still match the fp64 oracle within 2e-4); the inference path
// keeps its bf16 tcgen05 kernels and takes the trained weights through otif_proxy_create.
// C2 batch-32 step: 16.0 ms (SIMT, integer divisions) -> 4.0 ms (tcgen05, multiply-high
// divisors, coalesced K-contiguous staging with 16-B loads, 16-k stages at 2-3 CTAs per SM,
// tensor-tile split-K, parallel head reduce).
#include <math.h>
#include <stdlib.h>
#include <string.h>

#include <algorithm>
#include <type_traits>
#include <vector>

#include "common.cuh"

namespace otif {
namespace {

constexpr int BM = 64, BN = 64, BK = 16, GT = 256;

// ---- labels ----------------------------------------------------------------------------
__global__ void labels_kernel(const int32_t *__restrict__ boxes, int64_t nb, int n, int gh, int gw, int cell,
                              int frame_w, int frame_h, uint8_t *__restrict__ labels) {
    for (int64_t b = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; b < nb; b += (int64_t)gridDim.x * blockDim.x) {
        const int32_t *d = boxes + 5 * b;
        const int f = d[0];
        if (f < 0 || f >= n) continue;
        const int x0 = max(d[1], 0), y0 = max(d[2], 0), x1 = min(d[3], frame_w), y1 = min(d[4], frame_h);
        if (x0 >= x1 || y0 >= y1) continue;
        // cells [cx*cell, (cx+1)*cell) overlapping [x0, x1): cx in [x0/cell, (x1-1)/cell]
        for (int cy = y0 / cell; cy <= (y1 - 1) / cell && cy < gh; cy++)
            for (int cx = x0 / cell; cx <= (x1 - 1) / cell && cx < gw; cx++)
                labels[((int64_t)f * gh + cy) * gw + cx] = 1;
    }
}

// ---- generic SIMT GEMM -------------------------------------------------------------------
// Op supplies: a(m, k), b(k, n) (0 outside), store(m, n, value, split), and the layout flags
// A_KFAST / B_KFAST (true when consecutive k are contiguous in memory: the tile loaders
// then walk k fastest, otherwise m / n fastest) for coalesced loads.
template <class Op>
__global__ void __launch_bounds__(GT) sgemm_kernel(Op op, int M, int N, int K, int k_split) {
    __shared__ float As[BK][BM + 4];
    __shared__ float Bs[BK][BN + 4];
    const int tid = threadIdx.x, tx = tid & 15, ty = tid >> 4;
    const int m0 = blockIdx.x * BM, n0 = blockIdx.y * BN;
    const int kb = blockIdx.z * k_split, ke = min(K, kb + k_split);
    float acc[4][4] = {};
    for (int k0 = kb; k0 < ke; k0 += BK) {
#pragma unroll
        for (int i = 0; i < 4; i++) {
            const int e = tid + GT * i;
            const int kk = Op::A_KFAST ? (e & (BK - 1)) : (e / BM);
            const int mm = Op::A_KFAST ? (e / BK) : (e & (BM - 1));
            const int m = m0 + mm, k = k0 + kk;
            As[kk][mm] = (m < M && k < ke) ? op.a(m, k) : 0.f;
        }
#pragma unroll
        for (int i = 0; i < 4; i++) {
            const int e = tid + GT * i;
            const int kk = Op::B_KFAST ? (e & (BK - 1)) : (e / BN);
            const int nn = Op::B_KFAST ? (e / BK) : (e & (BN - 1));
            const int n = n0 + nn, k = k0 + kk;
            Bs[kk][nn] = (n < N && k < ke) ? op.b(k, n) : 0.f;
        }
        __syncthreads();
#pragma unroll
        for (int kk = 0; kk < BK; kk++) {
            float a[4], b[4];
#pragma unroll
            for (int i = 0; i < 4; i++) a[i] = As[kk][ty + 16 * i];
#pragma unroll
            for (int j = 0; j < 4; j++) b[j] = Bs[kk][tx + 16 * j];
#pragma unroll
            for (int i = 0; i < 4; i++)
#pragma unroll
                for (int j = 0; j < 4; j++) acc[i][j] = fmaf(a[i], b[j], acc[i][j]);
        }
        __syncthreads();
    }
#pragma unroll
    for (int i = 0; i < 4; i++)
#pragma unroll
        for (int j = 0; j < 4; j++) {
            const int m = m0 + ty + 16 * i, n = n0 + tx + 16 * j;
            if (m < M && n < N) op.store(m, n, acc[i][j], blockIdx.z);
        }
}


// ---- tcgen05 implicit GEMM (3xTF32) ------------------------------------------------------
// The same Op interface on the 5th-gen tensor cores.  fp32 operands are split into
// x = hi + lo with hi = tf32(x) (round to nearest) and lo = x - hi (exact in fp32); the
// product is accumulated in fp32 TMEM as hi·hi + hi·lo + lo·hi ("3xTF32"), which keeps
// the gradients at fp32 accuracy (the dropped lo·lo term is ~2^-22 relative).
// CTA: 256 threads load a 128 x 32 A chunk and a BN x 32 B chunk per stage (gathers
// through op.a / op.b, thread = (row, 4 consecutive k): one 16-B shared store per thread
// into the no-swizzle K-major core-matrix layout), 2 stages; warp 0 issues the 12 MMAs
// (M128 x BN x K8, kind::tf32) of a stage and commits them to the stage's "empty"
// barrier, so loads of chunk c+1 overlap the MMAs of chunk c.  Epilogue: tcgen05.ld
// (lane = row) -> op.store.  Split-K over blockIdx.z exactly like sgemm_kernel.
#ifndef OTIF_TC_K
#define OTIF_TC_K 16          // k per shared-memory stage (16: 3 CTAs per SM at BN = 128)
#endif
#ifndef OTIF_TC_MINB
#define OTIF_TC_MINB 2
#endif
constexpr int kTcThreads = 256, kTcM = 128, kTcK = OTIF_TC_K;

__device__ __forceinline__ float tf32_rna(float x) {
    uint32_t r;
    asm("cvt.rna.tf32.f32 %0, %1;" : "=r"(r) : "f"(x));
    return __uint_as_float(r);
}

__device__ __forceinline__ void umma_tf32_warp(uint32_t tmem_d, uint64_t adesc, uint64_t bdesc, uint32_t idesc,
                                               uint32_t accumulate) {
    asm volatile(
        "{\n\t.reg .pred p, e;\n\t"
        "setp.ne.b32 p, %4, 0;\n\t"
        "elect.sync _|e, 0xffffffff;\n\t"
        "@e tcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n\t}" ::"r"(tmem_d),
        "l"(adesc), "l"(bdesc), "r"(idesc), "r"(accumulate)
        : "memory");
}

// stage rows [0, R) x 32 k of one operand: thread t owns row t % R (R divides the CTA size)
// and k-groups t / R, t / R + 256 / R, ...; ctx = the row's context (op.a_row / op.b_row).
// Split into a load half (gathers into registers) and a store half (tf32 split + 16-B
// shared stores) so the kernel can keep the next chunks' gathers in flight (OTIF_TC_PREFETCH).
template <int R>
struct TcRowsRegs {
    static constexpr int kN = (kTcK / 4 + kTcThreads / R - 1) / (kTcThreads / R);
    float v[kN][4];
};
template <int R>
struct TcKfastRegs {
    static constexpr int kN = ((R / 8) * (kTcK / 16) + kTcThreads / 32 - 1) / (kTcThreads / 32);
    float v[kN][4];
};

template <int R, class Ctx, class F, class F4>
__device__ __forceinline__ void tc_load_operand(const Ctx &ctx, bool row_ok, F get, F4 get4, bool vec, int k0, int ke,
                                                TcRowsRegs<R> &g) {
    static_assert(kTcThreads % R == 0, "rows per thread");
    constexpr int kKG = kTcK / 4, kStep = kTcThreads / R, kIters = TcRowsRegs<R>::kN;
    if ((int)threadIdx.x / R >= kKG) return;   // more threads than (row, k-group) units
    // all the thread's loads first (kIters x 4 in flight: the gathers are latency-bound)
#pragma unroll
    for (int it = 0; it < kIters; it++) {
        const int kg = (int)threadIdx.x / R + it * kStep;
        const int kb4 = k0 + kg * 4;
        if (vec && row_ok && kg < kKG && kb4 + 4 <= ke) {
            get4(ctx, kb4, g.v[it]);   // four consecutive k with one index decomposition
        } else {
#pragma unroll
            for (int j = 0; j < 4; j++) {
                const int k = kb4 + j;
                g.v[it][j] = (row_ok && kg < kKG && k < ke) ? get(ctx, k) : 0.f;
            }
        }
    }
}

template <int R>
__device__ __forceinline__ void tc_store_operand(const TcRowsRegs<R> &g, uint8_t *hi, uint8_t *lo) {
    constexpr int kKG = kTcK / 4, kStep = kTcThreads / R, kIters = TcRowsRegs<R>::kN;
    const int r = threadIdx.x % R;
    if ((int)threadIdx.x / R >= kKG) return;
#pragma unroll
    for (int it = 0; it < kIters; it++) {
        const int kg = (int)threadIdx.x / R + it * kStep;
        if (kg >= kKG) continue;
        float h[4], l[4];
#pragma unroll
        for (int j = 0; j < 4; j++) { h[j] = tf32_rna(g.v[it][j]); l[j] = g.v[it][j] - h[j]; }
        const size_t off = ((size_t)kg * R + r) * 16;
        *reinterpret_cast<float4 *>(hi + off) = make_float4(h[0], h[1], h[2], h[3]);
        *reinterpret_cast<float4 *>(lo + off) = make_float4(l[0], l[1], l[2], l[3]);
    }
}

// K-contiguous operands (Op::*_KFAST): a warp stages 8 rows x 4 k-groups per unit (lane:
// row = l & 7, k-group = l >> 3), so each load instruction reads 64 contiguous bytes of 8
// rows (vs 32 scattered rows) and each 8-lane store phase hits 8 distinct 16-B bank
// groups.  Row contexts are recomputed per unit (mk: row -> context).
template <int R, class MK, class F, class F4>
__device__ __forceinline__ void tc_load_kfast(MK mk, int row0, int rows, F get, F4 get4, bool vec, int k0, int ke,
                                              TcKfastRegs<R> &g) {
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    constexpr int kGroups = kTcK / 16;                       // groups of 4 k-groups
    constexpr int kUnits = (R / 8) * kGroups, kWarps = kTcThreads / 32, kPerWarp = TcKfastRegs<R>::kN;
#pragma unroll
    for (int i = 0; i < kPerWarp; i++) {
        const int u = warp + i * kWarps;
        const int r = (u / kGroups) * 8 + (lane & 7), kg = (u % kGroups) * 4 + (lane >> 3);
        const bool ok = u < kUnits && r < rows;
        const auto q = mk(ok ? row0 + r : row0);
        const int kb4 = k0 + kg * 4;
        if (vec && ok && kb4 + 4 <= ke) {
            get4(q, kb4, g.v[i]);   // four consecutive k in one 16-B load
        } else {
#pragma unroll
            for (int j = 0; j < 4; j++) {
                const int k = kb4 + j;
                g.v[i][j] = (ok && k < ke) ? get(q, k) : 0.f;
            }
        }
    }
}

template <int R>
__device__ __forceinline__ void tc_store_kfast(const TcKfastRegs<R> &g, uint8_t *hi, uint8_t *lo) {
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    constexpr int kGroups = kTcK / 16;
    constexpr int kUnits = (R / 8) * kGroups, kWarps = kTcThreads / 32, kPerWarp = TcKfastRegs<R>::kN;
#pragma unroll
    for (int i = 0; i < kPerWarp; i++) {
        const int u = warp + i * kWarps;
        if (u >= kUnits) continue;
        const int r = (u / kGroups) * 8 + (lane & 7), kg = (u % kGroups) * 4 + (lane >> 3);
        float h[4], l[4];
#pragma unroll
        for (int j = 0; j < 4; j++) { h[j] = tf32_rna(g.v[i][j]); l[j] = g.v[i][j] - h[j]; }
        const size_t off = ((size_t)kg * R + r) * 16;
        *reinterpret_cast<float4 *>(hi + off) = make_float4(h[0], h[1], h[2], h[3]);
        *reinterpret_cast<float4 *>(lo + off) = make_float4(l[0], l[1], l[2], l[3]);
    }
}

#ifndef OTIF_TC_PREFETCH
#define OTIF_TC_PREFETCH 1    // 1: two register sets, chunk c+2's gathers issued while c+1's are in flight
#endif

template <class Op, int BN>
__global__ void __launch_bounds__(kTcThreads, OTIF_TC_MINB) tc_gemm_kernel(Op op, int M, int N, int K, int k_split) {
    extern __shared__ __align__(1024) uint8_t smem[];
    constexpr uint32_t kA = kTcM * kTcK * 4, kB = BN * kTcK * 4, kStage = 2 * kA + 2 * kB;
    __shared__ uint64_t full[2], empty[2], done;
    __shared__ uint32_t tslot;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int m0 = blockIdx.x * kTcM, n0 = blockIdx.y * BN;
    const int kb = blockIdx.z * k_split, ke = min(K, kb + k_split);
    if (threadIdx.x == 0) {
        for (int i = 0; i < 2; i++) { mbar_init(&full[i], kTcThreads); mbar_init(&empty[i], 1); }
        mbar_init(&done, 1);
        fence_barrier_init();
    }
    if (warp == 0) tmem_alloc(&tslot, BN < 32 ? 32 : BN);
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem = tslot;
    const uint32_t idesc = (1u << 4) | (2u << 7) | (2u << 10) | ((uint32_t)(BN >> 3) << 17) | ((uint32_t)(kTcM >> 4) << 24);
    const int nchunks = ke > kb ? (ke - kb + kTcK - 1) / kTcK : 0;
    const int am = m0 + (int)threadIdx.x % kTcM, bn = n0 + (int)threadIdx.x % BN;
    const bool a_ok = am < M, b_ok = bn < N;
    const typename Op::ARow actx = op.a_row(a_ok ? am : 0);
    const typename Op::BRow bctx = op.b_row(b_ok ? bn : 0);
    using ARegs = typename std::conditional<Op::A_KFAST, TcKfastRegs<kTcM>, TcRowsRegs<kTcM>>::type;
    using BRegs = typename std::conditional<Op::B_KFAST, TcKfastRegs<BN>, TcRowsRegs<BN>>::type;
    auto load = [&](int c, ARegs &ra, BRegs &rb) {
        const int k0 = kb + c * kTcK;
        if constexpr (Op::A_KFAST)
            tc_load_kfast<kTcM>([&](int m) { return op.a_row(m); }, m0, M - m0,
                                [&](const typename Op::ARow &q, int k) { return op.a_at(q, k); },
                                [&](const typename Op::ARow &q, int k, float *v) { op.a_at4(q, k, v); }, op.a_vec(),
                                k0, ke, ra);
        else
            tc_load_operand<kTcM>(actx, a_ok, [&](const typename Op::ARow &q, int k) { return op.a_at(q, k); },
                                  [&](const typename Op::ARow &q, int k, float *v) { op.a_at4(q, k, v); }, op.a_vec(),
                                  k0, ke, ra);
        if constexpr (Op::B_KFAST)
            tc_load_kfast<BN>([&](int n) { return op.b_row(n); }, n0, N - n0,
                              [&](const typename Op::BRow &q, int k) { return op.b_at(q, k); },
                              [&](const typename Op::BRow &q, int k, float *v) { op.b_at4(q, k, v); }, op.b_vec(), k0,
                              ke, rb);
        else
            tc_load_operand<BN>(bctx, b_ok, [&](const typename Op::BRow &q, int k) { return op.b_at(q, k); },
                                [&](const typename Op::BRow &q, int k, float *v) { op.b_at4(q, k, v); }, op.b_vec(),
                                k0, ke, rb);
    };
    // store chunk c's registers into its stage, hand the stage to the MMA warp; `next`
    // issues the gathers of a later chunk into the registers just freed (before warp 0
    // waits on the stage barrier), so they overlap the hand-off
    auto stage = [&](int c, ARegs &ra, BRegs &rb, int next) {
        const int st = c & 1;
        if (c >= 2) mbar_wait(&empty[st], ((c >> 1) - 1) & 1);   // the MMAs of chunk c-2 read this stage
        uint8_t *base = smem + (size_t)st * kStage;
        if constexpr (Op::A_KFAST) tc_store_kfast<kTcM>(ra, base, base + kA);
        else tc_store_operand<kTcM>(ra, base, base + kA);
        if constexpr (Op::B_KFAST) tc_store_kfast<BN>(rb, base + 2 * kA, base + 2 * kA + kB);
        else tc_store_operand<BN>(rb, base + 2 * kA, base + 2 * kA + kB);
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        mbar_arrive(&full[st]);
        if (next < nchunks) load(next, ra, rb);
        if (warp == 0) {
            mbar_wait(&full[st], (c >> 1) & 1);
            tc_fence_after();
            const uint32_t ah = smem_u32(base), al = ah + kA, bh = ah + 2 * kA, bl = bh + kB;
#pragma unroll
            for (int s = 0; s < kTcK / 8; s++) {
                const uint32_t ao = 2 * s * (kTcM * 16), bo = 2 * s * (BN * 16);
                const uint64_t dah = umma_desc(ah + ao, kTcM * 16, 128), dal = umma_desc(al + ao, kTcM * 16, 128);
                const uint64_t dbh = umma_desc(bh + bo, BN * 16, 128), dbl = umma_desc(bl + bo, BN * 16, 128);
                umma_tf32_warp(tmem, dal, dbh, idesc, (c > 0 || s > 0) ? 1u : 0u);
                umma_tf32_warp(tmem, dah, dbl, idesc, 1u);
                umma_tf32_warp(tmem, dah, dbh, idesc, 1u);
            }
            umma_commit_warp(&empty[st]);
        }
    };
#if OTIF_TC_PREFETCH >= 2
    {   // three register sets (A/B variant)
        ARegs ra0, ra1, ra2;
        BRegs rb0, rb1, rb2;
        if (nchunks > 0) load(0, ra0, rb0);
        if (nchunks > 1) load(1, ra1, rb1);
        if (nchunks > 2) load(2, ra2, rb2);
#pragma unroll 1
        for (int c = 0; c < nchunks; c += 3) {
            stage(c, ra0, rb0, c + 3);
            if (c + 1 < nchunks) stage(c + 1, ra1, rb1, c + 4);
            if (c + 2 < nchunks) stage(c + 2, ra2, rb2, c + 5);
        }
    }
#elif OTIF_TC_PREFETCH
    {
        ARegs ra0, ra1;
        BRegs rb0, rb1;
        if (nchunks > 0) load(0, ra0, rb0);
        if (nchunks > 1) load(1, ra1, rb1);
#pragma unroll 1
        for (int c = 0; c < nchunks; c += 2) {
            stage(c, ra0, rb0, c + 2);
            if (c + 1 < nchunks) stage(c + 1, ra1, rb1, c + 3);
        }
    }
#else
    {
        ARegs ra;
        BRegs rb;
#pragma unroll 1
        for (int c = 0; c < nchunks; c++) {
            load(c, ra, rb);
            stage(c, ra, rb, nchunks);
        }
    }
#endif
    if (warp == 0) umma_commit_warp(&done);
    mbar_wait(&done, 0);
    tc_fence_after();
    // epilogue: warp w reads lanes 32 (w & 3).. and columns [(w >> 2) BN/2, +BN/2)
    const int row = (warp & 3) * 32 + lane, m = m0 + row;
    constexpr int kHalf = BN / 2 < 32 ? BN : BN / 2;          // BN = 32: warps 0-3 take all columns
    const int c_lo = (warp >> 2) * kHalf, c_hi = c_lo + kHalf < BN ? c_lo + kHalf : BN;
#pragma unroll 1
    for (int cc = c_lo; cc < c_hi; cc += 32) {
        uint32_t v[32];
        if (nchunks > 0) {
            tmem_ld32(tmem + ((uint32_t)((warp & 3) * 32) << 16) + cc, v);
        } else {
#pragma unroll
            for (int j = 0; j < 32; j++) v[j] = 0u;
        }
        if (m < M)
            for (int j = 0; j < 32; j++) {
                const int n = n0 + cc + j;
                if (n < N) op.store(m, n, __uint_as_float(v[j]), blockIdx.z);
            }
    }
    tc_fence_before();
    __syncthreads();
    if (warp == 0) {
        tc_fence_after();
        tmem_dealloc(tmem, BN < 32 ? 32 : BN);
    }
}

struct ConvGeom {
    int H, W, Cin, Ho, Wo, Cout, k, stride, pad;
    // multiply-high divisors for the gathers' index math (set by with_divs on the host)
    FastDiv dHoWo, dWo, dHW, dW, dCin, dCout, dK, dStride;
};

static ConvGeom with_divs(ConvGeom g) {
    g.dHoWo = make_fastdiv((uint32_t)(g.Ho * g.Wo)); g.dWo = make_fastdiv((uint32_t)g.Wo);
    g.dHW = make_fastdiv((uint32_t)(g.H * g.W)); g.dW = make_fastdiv((uint32_t)g.W);
    g.dCin = make_fastdiv((uint32_t)g.Cin); g.dCout = make_fastdiv((uint32_t)g.Cout);
    g.dK = make_fastdiv((uint32_t)g.k); g.dStride = make_fastdiv((uint32_t)g.stride);
    return g;
}
__device__ __forceinline__ int dv(int n, const FastDiv &d) { return (int)fdiv((uint32_t)n, d); }

template <typename T>
__device__ __forceinline__ float act_in(const T *x, int64_t idx);
template <>
__device__ __forceinline__ float act_in<float>(const float *x, int64_t idx) { return x[idx]; }
template <>
__device__ __forceinline__ float act_in<uint8_t>(const uint8_t *x, int64_t idx) {
    return ((float)x[idx] - 128.f) * (1.f / 128.f);           // (u - 128) / 128, exact in fp32
}

// y[m = (f, oy, ox), co] = ReLU(Σ_k im2col(x)[m, k] W[co, k] + b[co]),  k = (kh, kw, ci)
template <typename T>
struct FwdOp {
    static constexpr bool A_KFAST = true, B_KFAST = true;
    const T *x;
    const float *w, *bias;
    float *y;
    ConvGeom g;
    int relu;
    // row contexts: the pixel of row m (A) / the weight row n (B) are fixed per thread in
    // tc_gemm_kernel, so their index math is done once
    struct ARow { int f, iy0, ix0; };
    __device__ ARow a_row(int m) const {
        const int f = dv(m, g.dHoWo), r = m - f * g.Ho * g.Wo, oy = dv(r, g.dWo), ox = r - oy * g.Wo;
        return {f, oy * g.stride - g.pad, ox * g.stride - g.pad};
    }
    __device__ float a_at(const ARow &q, int k) const {
        const int tap = dv(k, g.dCin), ci = k - tap * g.Cin, kh = dv(tap, g.dK), kw = tap - kh * g.k;
        const int iy = q.iy0 + kh, ix = q.ix0 + kw;
        if (iy < 0 || iy >= g.H || ix < 0 || ix >= g.W) return 0.f;
        return act_in<T>(x, (((int64_t)q.f * g.H + iy) * g.W + ix) * g.Cin + ci);
    }
    using BRow = const float *;
    __device__ BRow b_row(int n) const { return w + (int64_t)n * (g.k * g.k * g.Cin); }
    __device__ float b_at(BRow q, int k) const { return q[k]; }
    __device__ float a(int m, int k) const { return a_at(a_row(m), k); }
    __device__ float b(int k, int n) const { return b_at(b_row(n), k); }
    // 4 consecutive k (k % 4 == 0) in one 16-B load: same tap, consecutive channels when
    // Cin % 4 == 0 (fp32 activations); the weights rows are K = 9 Cin long
    __device__ bool a_vec() const { return sizeof(T) == 4 && g.Cin % 4 == 0 && (((uintptr_t)x) & 15) == 0; }
    __device__ bool b_vec() const { return (g.k * g.k * g.Cin) % 4 == 0 && (((uintptr_t)w) & 15) == 0; }
    __device__ void a_at4(const ARow &q, int k, float *v) const {
        if constexpr (sizeof(T) == 4) {
            const int tap = dv(k, g.dCin), ci = k - tap * g.Cin, kh = dv(tap, g.dK), kw = tap - kh * g.k;
            const int iy = q.iy0 + kh, ix = q.ix0 + kw;
            if (iy < 0 || iy >= g.H || ix < 0 || ix >= g.W) { v[0] = v[1] = v[2] = v[3] = 0.f; return; }
            const float4 t = *reinterpret_cast<const float4 *>(
                reinterpret_cast<const float *>(x) + (((int64_t)q.f * g.H + iy) * g.W + ix) * g.Cin + ci);
            v[0] = t.x; v[1] = t.y; v[2] = t.z; v[3] = t.w;
        } else {
            for (int j = 0; j < 4; j++) v[j] = a_at(q, k + j);
        }
    }
    __device__ void b_at4(BRow q, int k, float *v) const {
        const float4 t = *reinterpret_cast<const float4 *>(q + k);
        v[0] = t.x; v[1] = t.y; v[2] = t.z; v[3] = t.w;
    }
    __device__ void store(int m, int n, float v, int) const {
        v += bias[n];
        y[(int64_t)m * g.Cout + n] = relu ? fmaxf(v, 0.f) : v;
    }
};

// dx[m = (f, iy, ix), ci] = Σ_{kh, kw, co} dy[f, oy, ox, co] W[co, kh, kw, ci] where
// iy = oy*s - pad + kh, then ⊙ [x_post > 0] (the ReLU of the layer below): the result is
// that layer's pre-activation gradient.  k = (kh, kw, co).
struct DgradOp {
    static constexpr bool A_KFAST = true, B_KFAST = false;
    const float *dy, *w, *xpost;
    float *dx;
    ConvGeom g;
    struct ARow { int f, ty0, tx0; };
    __device__ ARow a_row(int m) const {
        const int f = dv(m, g.dHW), r = m - f * g.H * g.W, iy = dv(r, g.dW), ix = r - iy * g.W;
        return {f, iy + g.pad, ix + g.pad};
    }
    __device__ float a_at(const ARow &q, int k) const {
        const int tap = dv(k, g.dCout), co = k - tap * g.Cout, kh = dv(tap, g.dK), kw = tap - kh * g.k;
        const int ty = q.ty0 - kh, tx = q.tx0 - kw;
        if (ty < 0 || tx < 0) return 0.f;
        const int oy = dv(ty, g.dStride), ox = dv(tx, g.dStride);
        if (oy * g.stride != ty || ox * g.stride != tx || oy >= g.Ho || ox >= g.Wo) return 0.f;
        return dy[(((int64_t)q.f * g.Ho + oy) * g.Wo + ox) * g.Cout + co];
    }
    using BRow = int;
    __device__ BRow b_row(int n) const { return n; }
    __device__ float b_at(BRow n, int k) const {
        const int tap = dv(k, g.dCout), co = k - tap * g.Cout;
        return w[((int64_t)co * g.k * g.k + tap) * g.Cin + n];
    }
    // 4 consecutive k = 4 consecutive output channels of one tap (Cout % 4 == 0)
    __device__ bool a_vec() const { return g.Cout % 4 == 0 && (((uintptr_t)dy) & 15) == 0; }
    __device__ bool b_vec() const { return false; }
    __device__ void a_at4(const ARow &q, int k, float *v) const {
        const int tap = dv(k, g.dCout), co = k - tap * g.Cout, kh = dv(tap, g.dK), kw = tap - kh * g.k;
        const int ty = q.ty0 - kh, tx = q.tx0 - kw;
        v[0] = v[1] = v[2] = v[3] = 0.f;
        if (ty < 0 || tx < 0) return;
        const int oy = dv(ty, g.dStride), ox = dv(tx, g.dStride);
        if (oy * g.stride != ty || ox * g.stride != tx || oy >= g.Ho || ox >= g.Wo) return;
        const float4 t = *reinterpret_cast<const float4 *>(dy + (((int64_t)q.f * g.Ho + oy) * g.Wo + ox) * g.Cout + co);
        v[0] = t.x; v[1] = t.y; v[2] = t.z; v[3] = t.w;
    }
    __device__ void b_at4(BRow n, int k, float *v) const {
        for (int j = 0; j < 4; j++) v[j] = b_at(n, k + j);
    }
    __device__ float a(int m, int k) const { return a_at(a_row(m), k); }
    __device__ float b(int k, int n) const { return b_at(b_row(n), k); }
    __device__ void store(int m, int n, float v, int) const {
        const int64_t i = (int64_t)m * g.Cin + n;
        dx[i] = xpost[i] > 0.f ? v : 0.f;
    }
};

// Stride-2 dgrad split by the parity (py, px) of the input pixel: only the taps with
// kh = py + 1 (mod 2) and kw = px + 1 (mod 2) reach an output pixel (ty = iy + 1 - kh even),
// so each class is a GEMM over ntap = 1, 2, 2 or 4 taps instead of 9 with 3/4 zeros
// (M = that class's pixels, K = ntap x Cout).  Same sums as DgradOp without its zero terms.
struct DgradParOp {
    static constexpr bool A_KFAST = true, B_KFAST = false;
    const float *dy, *w, *xpost;
    float *dx;
    ConvGeom g;
    int py, px, Hc, Wc, ntap;
    int tkh[4], tkw[4];
    FastDiv dHWc, dWc, dCout;
    struct ARow { int f, ty0, tx0; int64_t pix; };
    __device__ ARow a_row(int m) const {
        const int f = dv(m, dHWc), r = m - f * Hc * Wc, iyc = dv(r, dWc), ixc = r - iyc * Wc;
        const int iy = 2 * iyc + py, ix = 2 * ixc + px;
        return {f, iy + g.pad, ix + g.pad, ((int64_t)f * g.H + iy) * g.W + ix};
    }
    __device__ float a_at(const ARow &q, int k) const {
        const int t = dv(k, dCout), co = k - t * g.Cout;
        const int ty = q.ty0 - tkh[t], tx = q.tx0 - tkw[t];
        if (ty < 0 || tx < 0) return 0.f;
        const int oy = ty >> 1, ox = tx >> 1;
        if (oy >= g.Ho || ox >= g.Wo) return 0.f;
        return dy[(((int64_t)q.f * g.Ho + oy) * g.Wo + ox) * g.Cout + co];
    }
    using BRow = int;
    __device__ BRow b_row(int n) const { return n; }
    __device__ float b_at(BRow n, int k) const {
        const int t = dv(k, dCout), co = k - t * g.Cout;
        return w[((int64_t)co * g.k * g.k + tkh[t] * g.k + tkw[t]) * g.Cin + n];
    }
    __device__ float a(int m, int k) const { return a_at(a_row(m), k); }
    __device__ float b(int k, int n) const { return b_at(b_row(n), k); }
    __device__ bool a_vec() const { return g.Cout % 4 == 0 && (((uintptr_t)dy) & 15) == 0; }
    __device__ bool b_vec() const { return false; }
    __device__ void a_at4(const ARow &q, int k, float *v) const {
        const int t = dv(k, dCout), co = k - t * g.Cout;
        const int ty = q.ty0 - tkh[t], tx = q.tx0 - tkw[t];
        v[0] = v[1] = v[2] = v[3] = 0.f;
        if (ty < 0 || tx < 0) return;
        const int oy = ty >> 1, ox = tx >> 1;
        if (oy >= g.Ho || ox >= g.Wo) return;
        const float4 x4 = *reinterpret_cast<const float4 *>(dy + (((int64_t)q.f * g.Ho + oy) * g.Wo + ox) * g.Cout + co);
        v[0] = x4.x; v[1] = x4.y; v[2] = x4.z; v[3] = x4.w;
    }
    __device__ void b_at4(BRow n, int k, float *v) const {
        for (int j = 0; j < 4; j++) v[j] = b_at(n, k + j);
    }
    __device__ void store(int m, int n, float v, int) const {
        const int f = dv(m, dHWc), r = m - f * Hc * Wc, iyc = dv(r, dWc), ixc = r - iyc * Wc;
        const int64_t i = (((int64_t)f * g.H + 2 * iyc + py) * g.W + 2 * ixc + px) * g.Cin + n;
        dx[i] = xpost[i] > 0.f ? v : 0.f;
    }
};

// [dW | db][co, kk] = Σ_p dy[p, co] · (kk < K ? im2col(x)[p, kk] : 1), split over p.
template <typename T>
struct WgradOp {
    static constexpr bool A_KFAST = false, B_KFAST = false;
    const float *dy;
    const T *x;
    float *part;        // [split][Cout][K + 1]
    ConvGeom g;
    int Kw;             // k*k*Cin
    using ARow = int;
    __device__ ARow a_row(int m) const { return m; }
    __device__ float a_at(ARow co, int p) const { return dy[(int64_t)p * g.Cout + co]; }
    struct BRow { int bias, ci, kh, kw; };
    __device__ BRow b_row(int kk) const {
        if (kk == Kw) return {1, 0, 0, 0};
        const int tap = dv(kk, g.dCin), kh = dv(tap, g.dK);
        return {0, kk - tap * g.Cin, kh, tap - kh * g.k};
    }
    __device__ float b_at(const BRow &q, int p) const {
        if (q.bias) return 1.f;
        const int f = dv(p, g.dHoWo), r = p - f * g.Ho * g.Wo, oy = dv(r, g.dWo), ox = r - oy * g.Wo;
        const int iy = oy * g.stride - g.pad + q.kh, ix = ox * g.stride - g.pad + q.kw;
        if (iy < 0 || iy >= g.H || ix < 0 || ix >= g.W) return 0.f;
        return act_in<T>(x, (((int64_t)f * g.H + iy) * g.W + ix) * g.Cin + q.ci);
    }
    __device__ float a(int m, int p) const { return a_at(a_row(m), p); }
    __device__ float b(int p, int kk) const { return b_at(b_row(kk), p); }
    __device__ bool a_vec() const { return false; }
    __device__ bool b_vec() const { return true; }   // 4 consecutive pixels: one decomposition, then steps
    __device__ void a_at4(ARow q, int k, float *v) const { for (int j = 0; j < 4; j++) v[j] = a_at(q, k + j); }
    __device__ void b_at4(const BRow &q, int p, float *v) const {
        if (q.bias) { v[0] = v[1] = v[2] = v[3] = 1.f; return; }
        int f = dv(p, g.dHoWo), r = p - f * g.Ho * g.Wo, oy = dv(r, g.dWo), ox = r - oy * g.Wo;
#pragma unroll
        for (int j = 0; j < 4; j++) {
            const int iy = oy * g.stride - g.pad + q.kh, ix = ox * g.stride - g.pad + q.kw;
            v[j] = (iy < 0 || iy >= g.H || ix < 0 || ix >= g.W)
                       ? 0.f
                       : act_in<T>(x, (((int64_t)f * g.H + iy) * g.W + ix) * g.Cin + q.ci);
            if (++ox == g.Wo) { ox = 0; if (++oy == g.Ho) { oy = 0; f++; } }
        }
    }
    __device__ void store(int m, int n, float v, int split) const {
        part[((int64_t)split * g.Cout + m) * (Kw + 1) + n] = v;
    }
};

// fixed-order sum of the split partials into the blob: W[co][kk] then b[co]
__global__ void wgrad_reduce_kernel(const float *__restrict__ part, int splits, int cout, int kw,
                                    float *__restrict__ grad) {
    const int64_t total = (int64_t)cout * (kw + 1);
    for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < total; e += (int64_t)gridDim.x * blockDim.x) {
        float s = 0.f;
        for (int sp = 0; sp < splits; sp++) s += part[(int64_t)sp * total + e];
        const int co = (int)(e / (kw + 1)), kk = (int)(e - (int64_t)co * (kw + 1));
        if (kk < kw)
            grad[(int64_t)co * kw + kk] = s;
        else
            grad[(int64_t)cout * kw + co] = s;
    }
}

// D2 + sigmoid + BCE (reading R26), warp per cell (grid-stride, fixed assignment):
// z = b2 + Σ_c a[c] w2[c]; loss += softplus(z) - y z; dz = (sigmoid(z) - y) / M;
// d_pre[c] = dz w2[c] [a[c] > 0]; per-warp partials of Σ dz a[c] (dW2), Σ dz (db2), loss.
constexpr int kHeadWarps = 8;
__global__ void __launch_bounds__(kHeadWarps * 32) head_kernel(const float *__restrict__ act, const float *__restrict__ w2,
                                                               const uint8_t *__restrict__ labels, int64_t M, int dec,
                                                               float *__restrict__ dpre, float *__restrict__ part) {
    const int lane = threadIdx.x & 31;
    const int64_t gw = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    const float b2 = w2[dec];
    float dws[8] = {0, 0, 0, 0, 0, 0, 0, 0};      // channels lane + 32 i, dec <= 256
    float dbs = 0.f, ls = 0.f;
    const float invM = 1.f / (float)M;
    for (int64_t cidx = gw; cidx < M; cidx += nw) {
        const float *a = act + cidx * dec;
        float z = 0.f;
        for (int c = lane; c < dec; c += 32) z = fmaf(a[c], w2[c], z);
        for (int s = 16; s > 0; s >>= 1) z += __shfl_xor_sync(0xffffffffu, z, s);
        z += b2;
        const float y = labels[cidx] ? 1.f : 0.f;
        const float sp = z > 0.f ? z + log1pf(expf(-z)) : log1pf(expf(z));
        const float dz = (1.f / (1.f + expf(-z)) - y) * invM;
        ls += sp - y * z;
        dbs += dz;
#pragma unroll
        for (int i = 0; i < 8; i++) {
            const int c = lane + 32 * i;
            if (c < dec) {
                const float av = a[c];
                dws[i] = fmaf(dz, av, dws[i]);
                dpre[cidx * dec + c] = av > 0.f ? dz * w2[c] : 0.f;
            }
        }
    }
    float *o = part + gw * (dec + 2);
#pragma unroll
    for (int i = 0; i < 8; i++) {
        const int c = lane + 32 * i;
        if (c < dec) o[c] = dws[i];
    }
    if (lane == 0) {
        o[dec] = dbs;
        o[dec + 1] = ls;
    }
}

// fixed-order reduction of the head partials -> grad (W2, b2) and the mean loss: one CTA
// per column, each thread a fixed strided subset, then a fixed shared-memory tree
// (deterministic: the order never depends on scheduling)
__global__ void __launch_bounds__(256) head_reduce_kernel(const float *__restrict__ part, int64_t nwarps, int dec,
                                                          int64_t M, float *__restrict__ grad_w2,
                                                          float *__restrict__ loss) {
    __shared__ float red[256];
    const int c = blockIdx.x;
    float s = 0.f;
    for (int64_t w = threadIdx.x; w < nwarps; w += blockDim.x) s += part[w * (dec + 2) + c];
    red[threadIdx.x] = s;
    __syncthreads();
    for (int h = 128; h > 0; h >>= 1) {
        if ((int)threadIdx.x < h) red[threadIdx.x] += red[threadIdx.x + h];
        __syncthreads();
    }
    if (threadIdx.x == 0) {
        if (c <= dec)
            grad_w2[c] = red[0];                  // W2[0..dec-1], then b2
        else
            *loss = red[0] / (float)M;
    }
}

__global__ void adam_kernel(float *__restrict__ w, float *__restrict__ m, float *__restrict__ v,
                            const float *__restrict__ g, int64_t count, float lr, float b1, float b2, float eps,
                            float c1, float c2) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < count; i += (int64_t)gridDim.x * blockDim.x) {
        const float gi = g[i];
        const float mi = b1 * m[i] + (1.f - b1) * gi;
        const float vi = b2 * v[i] + (1.f - b2) * gi * gi;
        m[i] = mi;
        v[i] = vi;
        w[i] -= lr * (mi / c1) / (sqrtf(vi / c2) + eps);
    }
}

// 1 = tcgen05 3xTF32 (default), 0 = SIMT fp32 (A/B builds: nvcc -DOTIF_TRAIN_SIMT)
static int train_tc() {
#ifdef OTIF_TRAIN_SIMT
    return 0;
#else
    return 1;
#endif
}

template <class Op>
otif_status run_gemm(const Op &op, int64_t M, int64_t N, int64_t K, int splits, cudaStream_t stream) {
    if (M <= 0 || N <= 0) return OTIF_OK;
    if (train_tc()) {
        const int64_t k_split = round_up(cdiv(K, splits), kTcK);
        if (N <= 32) {
            constexpr int BNv = 32;
            const size_t smem = 2 * (2 * (size_t)kTcM * kTcK * 4 + 2 * (size_t)BNv * kTcK * 4);
            OTIF_CUDA(cudaFuncSetAttribute(tc_gemm_kernel<Op, BNv>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
            const dim3 grid((unsigned)cdiv(M, kTcM), (unsigned)cdiv(N, BNv), (unsigned)splits);
            tc_gemm_kernel<Op, BNv><<<grid, kTcThreads, smem, stream>>>(op, (int)M, (int)N, (int)K, (int)k_split);
        } else if (N <= 64) {
            constexpr int BNv = 64;
            const size_t smem = 2 * (2 * (size_t)kTcM * kTcK * 4 + 2 * (size_t)BNv * kTcK * 4);
            OTIF_CUDA(cudaFuncSetAttribute(tc_gemm_kernel<Op, BNv>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
            const dim3 grid((unsigned)cdiv(M, kTcM), (unsigned)cdiv(N, BNv), (unsigned)splits);
            tc_gemm_kernel<Op, BNv><<<grid, kTcThreads, smem, stream>>>(op, (int)M, (int)N, (int)K, (int)k_split);
        } else {
            constexpr int BNv = 128;
            const size_t smem = 2 * (2 * (size_t)kTcM * kTcK * 4 + 2 * (size_t)BNv * kTcK * 4);
            OTIF_CUDA(cudaFuncSetAttribute(tc_gemm_kernel<Op, BNv>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
            const dim3 grid((unsigned)cdiv(M, kTcM), (unsigned)cdiv(N, BNv), (unsigned)splits);
            tc_gemm_kernel<Op, BNv><<<grid, kTcThreads, smem, stream>>>(op, (int)M, (int)N, (int)K, (int)k_split);
        }
        OTIF_LAUNCH_CHECK();
        return OTIF_OK;
    }
    const int64_t k_split = round_up(cdiv(K, splits), BK);
    const dim3 grid((unsigned)cdiv(M, BM), (unsigned)cdiv(N, BN), (unsigned)splits);
    sgemm_kernel<Op><<<grid, GT, 0, stream>>>(op, (int)M, (int)N, (int)K, (int)k_split);
    OTIF_LAUNCH_CHECK();
    return OTIF_OK;
}

}  // namespace
}  // namespace otif

using namespace otif;

struct otif_trainer {
    otif_proxy_desc d;
    int max_batch = 0;
    int sms = 0;
    int cin[7], cout[7], ks[7], stride[7], hs[8], ws[8];
    size_t woff[7];
    size_t n_weights = 0;
    float *w = nullptr, *m = nullptr, *v = nullptr, *grad = nullptr;
    float *act[8] = {};          // act[1..6] fp32 NHWC post-ReLU; act[0] is the caller's u8 image
    float *dbuf[2] = {};         // pre-activation gradients, ping-pong
    float *part = nullptr;       // split-K / head partials
    size_t part_floats = 0;
    int64_t head_warps = 0;
    int step = 0;
};

#ifndef OTIF_WGRAD_WAVES
#define OTIF_WGRAD_WAVES 3     // split-K CTAs per SM targeted by the weight-gradient GEMMs
#endif
static int wgrad_splits(const otif_trainer *t, int L, int n) {
    const int64_t pixels = (int64_t)n * t->hs[L + 1] * t->ws[L + 1];
    const int64_t kw1 = (int64_t)t->ks[L] * t->ks[L] * t->cin[L] + 1;
    // output tiles of the GEMM kernel in use (tcgen05: 128 x 32/64/128; SIMT: 64 x 64)
    const int64_t tiles = train_tc() ? cdiv(t->cout[L], kTcM) * cdiv(kw1, kw1 <= 32 ? 32 : kw1 <= 64 ? 64 : 128)
                                     : cdiv(t->cout[L], BM) * cdiv(kw1, BN);
    int64_t s = cdiv(OTIF_WGRAD_WAVES * (int64_t)t->sms, tiles);
    s = std::min<int64_t>(s, std::max<int64_t>(1, pixels / 256));
    return (int)std::max<int64_t>(1, std::min<int64_t>(s, 512));
}

extern "C" otif_status otif_cell_labels(const int32_t *boxes, int64_t nb, int32_t n, int32_t gh, int32_t gw,
                                        const otif_grid_desc *g, uint8_t *labels, cudaStream_t stream) {
    OTIF_REQUIRE(g && labels && (boxes || nb == 0), "otif_cell_labels: NULL argument");
    OTIF_REQUIRE(n >= 0 && gh > 0 && gw > 0 && nb >= 0 && g->cell > 0 && g->frame_w > 0 && g->frame_h > 0,
                 "otif_cell_labels: bad sizes");
    otif_status st = check_device(nullptr);
    if (st != OTIF_OK) return st;
    if (n == 0) return OTIF_OK;
    OTIF_CUDA(cudaMemsetAsync(labels, 0, (size_t)n * gh * gw, stream));
    if (nb == 0) return OTIF_OK;
    labels_kernel<<<(unsigned)std::min<int64_t>(cdiv(nb, 256), 4096), 256, 0, stream>>>(
        boxes, nb, n, gh, gw, g->cell, g->frame_w, g->frame_h, labels);
    OTIF_LAUNCH_CHECK();
    return OTIF_OK;
}

extern "C" otif_status otif_adam_step(float *w, float *m, float *v, const float *g, int64_t count, int32_t t, float lr,
                                      float b1, float b2, float eps, cudaStream_t stream) {
    OTIF_REQUIRE(count >= 0 && t >= 1, "otif_adam_step: count=%lld t=%d", (long long)count, t);
    if (count == 0) return OTIF_OK;
    OTIF_REQUIRE(w && m && v && g, "otif_adam_step: NULL argument");
    int sms = 0;
    otif_status st = check_device(&sms);
    if (st != OTIF_OK) return st;
    const float c1 = (float)(1.0 - pow((double)b1, (double)t)), c2 = (float)(1.0 - pow((double)b2, (double)t));
    adam_kernel<<<(unsigned)std::min<int64_t>(cdiv(count, 256), (int64_t)sms * 8), 256, 0, stream>>>(
        w, m, v, g, count, lr, b1, b2, eps, c1, c2);
    OTIF_LAUNCH_CHECK();
    return OTIF_OK;
}

extern "C" otif_status otif_trainer_create(const otif_proxy_desc *d, const float *weights, size_t n_weights,
                                           int32_t max_batch, otif_trainer **out) {
    OTIF_REQUIRE(d && weights && out, "otif_trainer_create: NULL argument");
    OTIF_REQUIRE(d->in_h > 0 && d->in_w > 0 && d->n_strided >= 1 && d->n_strided <= 5 && max_batch >= 1,
                 "otif_trainer_create: in %dx%d n_strided %d max_batch %d", d->in_h, d->in_w, d->n_strided, max_batch);
    for (int i = 0; i < 5; i++) OTIF_REQUIRE(d->enc[i] > 0, "otif_trainer_create: enc[%d]=%d", i, d->enc[i]);
    OTIF_REQUIRE(d->dec > 0 && d->dec <= 256, "otif_trainer_create: dec=%d (1..256)", d->dec);
    int sms = 0;
    otif_status st = check_device(&sms);
    if (st != OTIF_OK) return st;
    otif_trainer *t = new otif_trainer();
    t->d = *d;
    t->max_batch = max_batch;
    t->sms = sms;
    int c = 3;
    for (int L = 0; L < 7; L++) {
        t->cin[L] = c;
        t->cout[L] = L < 5 ? d->enc[L] : (L == 5 ? d->dec : 1);
        t->ks[L] = L == 6 ? 1 : 3;
        t->stride[L] = (L < 5 && L < d->n_strided) ? 2 : 1;
        c = t->cout[L];
    }
    t->hs[0] = d->in_h;
    t->ws[0] = d->in_w;
    size_t off = 0, max_act = 0;
    for (int L = 0; L < 7; L++) {
        t->hs[L + 1] = (t->hs[L] + t->stride[L] - 1) / t->stride[L];
        t->ws[L + 1] = (t->ws[L] + t->stride[L] - 1) / t->stride[L];
        t->woff[L] = off;
        off += (size_t)t->cout[L] * t->ks[L] * t->ks[L] * t->cin[L] + t->cout[L];
        if (L < 6) max_act = std::max(max_act, (size_t)max_batch * t->hs[L + 1] * t->ws[L + 1] * t->cout[L]);
    }
    t->n_weights = off;
    if (n_weights != off) {
        delete t;
        set_error("otif_trainer_create: n_weights %zu != %zu", n_weights, off);
        return OTIF_EINVAL;
    }
    // partial buffers: max over layers of splits * Cout * (K + 1), and the head partials
    size_t part = 0;
    for (int L = 0; L < 6; L++) {
        const size_t kw = (size_t)t->ks[L] * t->ks[L] * t->cin[L];
        part = std::max(part, (size_t)wgrad_splits(t, L, max_batch) * t->cout[L] * (kw + 1));
    }
    t->head_warps = (int64_t)sms * 4 * kHeadWarps;
    part = std::max(part, (size_t)t->head_warps * (t->d.dec + 2));
    t->part_floats = part;
    bool ok = cudaMalloc(&t->w, off * 4) == cudaSuccess && cudaMalloc(&t->m, off * 4) == cudaSuccess &&
              cudaMalloc(&t->v, off * 4) == cudaSuccess && cudaMalloc(&t->grad, off * 4) == cudaSuccess &&
              cudaMalloc(&t->part, part * 4) == cudaSuccess && cudaMalloc(&t->dbuf[0], max_act * 4) == cudaSuccess &&
              cudaMalloc(&t->dbuf[1], max_act * 4) == cudaSuccess;
    for (int L = 1; L <= 6 && ok; L++)
        ok = cudaMalloc(&t->act[L], (size_t)max_batch * t->hs[L] * t->ws[L] * t->cout[L - 1] * 4) == cudaSuccess;
    if (!ok) {
        otif_trainer_destroy(t);
        set_error("otif_trainer_create: device allocation failed");
        return OTIF_ENOMEM;
    }
    if (cudaMemcpy(t->w, weights, off * 4, cudaMemcpyHostToDevice) != cudaSuccess ||
        cudaMemset(t->m, 0, off * 4) != cudaSuccess || cudaMemset(t->v, 0, off * 4) != cudaSuccess ||
        cudaMemset(t->grad, 0, off * 4) != cudaSuccess) {
        otif_trainer_destroy(t);
        set_error("otif_trainer_create: upload failed");
        return OTIF_ECUDA;
    }
    *out = t;
    return OTIF_OK;
}

extern "C" void otif_trainer_destroy(otif_trainer *t) {
    if (!t) return;
    cudaFree(t->w);
    cudaFree(t->m);
    cudaFree(t->v);
    cudaFree(t->grad);
    cudaFree(t->part);
    for (int i = 0; i < 2; i++) cudaFree(t->dbuf[i]);
    for (int L = 1; L <= 6; L++) cudaFree(t->act[L]);
    delete t;
}

extern "C" otif_status otif_trainer_params(const otif_trainer *t, float **weights, float **grads, size_t *n_weights,
                                           int32_t *gh, int32_t *gw) {
    OTIF_REQUIRE(t, "otif_trainer_params: NULL trainer");
    if (weights) *weights = t->w;
    if (grads) *grads = t->grad;
    if (n_weights) *n_weights = t->n_weights;
    if (gh) *gh = t->hs[7];
    if (gw) *gw = t->ws[7];
    return OTIF_OK;
}

extern "C" otif_status otif_trainer_backward(otif_trainer *t, const uint8_t *img, const uint8_t *labels, int32_t n,
                                             float *loss, cudaStream_t stream) {
    OTIF_REQUIRE(t && img && labels && loss, "otif_trainer_backward: NULL argument");
    OTIF_REQUIRE(n >= 1 && n <= t->max_batch, "otif_trainer_backward: n=%d (1..%d)", n, t->max_batch);
    otif_status st = check_device(nullptr);
    if (st != OTIF_OK) return st;
    auto geom = [&](int L) {
        ConvGeom g;
        g.H = t->hs[L]; g.W = t->ws[L]; g.Cin = t->cin[L]; g.Ho = t->hs[L + 1]; g.Wo = t->ws[L + 1];
        g.Cout = t->cout[L]; g.k = t->ks[L]; g.stride = t->stride[L]; g.pad = (t->ks[L] - 1) / 2;
        return with_divs(g);
    };
    // forward E1..D1 (D2 lives in the head kernel)
    for (int L = 0; L < 6; L++) {
        const ConvGeom g = geom(L);
        const float *wl = t->w + t->woff[L];
        const float *bl = wl + (size_t)g.Cout * g.k * g.k * g.Cin;
        const int64_t M = (int64_t)n * g.Ho * g.Wo, K = (int64_t)g.k * g.k * g.Cin;
        if (L == 0) {
            FwdOp<uint8_t> op{img, wl, bl, t->act[1], g, 1};
            st = run_gemm(op, M, g.Cout, K, 1, stream);
        } else {
            FwdOp<float> op{t->act[L], wl, bl, t->act[L + 1], g, 1};
            st = run_gemm(op, M, g.Cout, K, 1, stream);
        }
        if (st != OTIF_OK) return st;
    }
    // head: loss, D2 gradient, D1 pre-activation gradient
    const int dec = t->cout[5];
    const int64_t cells = (int64_t)n * t->hs[7] * t->ws[7];
    head_kernel<<<(unsigned)(t->head_warps / kHeadWarps), kHeadWarps * 32, 0, stream>>>(
        t->act[6], t->w + t->woff[6], labels, cells, dec, t->dbuf[0], t->part);
    OTIF_LAUNCH_CHECK();
    head_reduce_kernel<<<(unsigned)(dec + 2), 256, 0, stream>>>(t->part, t->head_warps, dec, cells, t->grad + t->woff[6], loss);
    OTIF_LAUNCH_CHECK();
    // backward D1 .. E1
    int cur = 0;
    for (int L = 5; L >= 0; L--) {
        const ConvGeom g = geom(L);
        const int kw = g.k * g.k * g.Cin;
        const int64_t P = (int64_t)n * g.Ho * g.Wo;
        const int splits = wgrad_splits(t, L, n);
        if (L == 0) {
            WgradOp<uint8_t> op{t->dbuf[cur], img, t->part, g, kw};
            st = run_gemm(op, g.Cout, kw + 1, P, splits, stream);
        } else {
            WgradOp<float> op{t->dbuf[cur], t->act[L], t->part, g, kw};
            st = run_gemm(op, g.Cout, kw + 1, P, splits, stream);
        }
        if (st != OTIF_OK) return st;
        wgrad_reduce_kernel<<<(unsigned)std::min<int64_t>(cdiv((int64_t)g.Cout * (kw + 1), 256), 4096), 256, 0,
                              stream>>>(t->part, splits, g.Cout, kw, t->grad + t->woff[L]);
        OTIF_LAUNCH_CHECK();
        if (L > 0) {
            if (g.stride == 2 && g.k == 3 && g.pad == 1 && train_tc()) {
                // four parity classes of input pixels, each with its own tap subset
                for (int py = 0; py < 2; py++)
                    for (int px = 0; px < 2; px++) {
                        DgradParOp op;
                        op.dy = t->dbuf[cur]; op.w = t->w + t->woff[L]; op.xpost = t->act[L]; op.dx = t->dbuf[cur ^ 1];
                        op.g = g; op.py = py; op.px = px;
                        op.Hc = (g.H - py + 1) / 2; op.Wc = (g.W - px + 1) / 2;
                        op.ntap = 0;
                        for (int kh = 0; kh < 3; kh++)
                            for (int kw = 0; kw < 3; kw++)
                                if (((py + 1 - kh) & 1) == 0 && ((px + 1 - kw) & 1) == 0) {
                                    op.tkh[op.ntap] = kh; op.tkw[op.ntap] = kw; op.ntap++;
                                }
                        op.dHWc = make_fastdiv((uint32_t)(op.Hc * op.Wc)); op.dWc = make_fastdiv((uint32_t)op.Wc);
                        op.dCout = make_fastdiv((uint32_t)g.Cout);
                        const int64_t Mc = (int64_t)n * op.Hc * op.Wc;
                        if (Mc == 0) continue;
                        st = run_gemm(op, Mc, g.Cin, (int64_t)op.ntap * g.Cout, 1, stream);
                        if (st != OTIF_OK) return st;
                    }
            } else {
                DgradOp op{t->dbuf[cur], t->w + t->woff[L], t->act[L], t->dbuf[cur ^ 1], g};
                st = run_gemm(op, (int64_t)n * g.H * g.W, g.Cin, (int64_t)g.k * g.k * g.Cout, 1, stream);
                if (st != OTIF_OK) return st;
            }
            cur ^= 1;
        }
    }
    return OTIF_OK;
}

extern "C" otif_status otif_trainer_adam(otif_trainer *t, float lr, cudaStream_t stream) {
    OTIF_REQUIRE(t, "otif_trainer_adam: NULL trainer");
    t->step++;
    return otif_adam_step(t->w, t->m, t->v, t->grad, (int64_t)t->n_weights, t->step, lr, 0.9f, 0.999f, 1e-8f,
                          stream);
}
