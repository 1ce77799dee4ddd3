// Microbenchmark + layout check: tcgen05.mma kind::f16 with A in TMEM ("TS"): A rows
// written by tcgen05.st (lane = row, 32-bit column = two consecutive K elements), B in
// shared memory (no-swizzle K-major core matrices).  Checks D against a host GEMM and
// measures clk per MMA for N = 32 / 64 (vs the SS rates of mma_rate.cu).
#include <cstdio>
#include <cstdlib>
#include <cuda_fp16.h>
#include <cuda_runtime.h>
#include "../../paper_conf_sigmod_bastanim22_b200/csrc/common.cuh"
using namespace otif;

__device__ __forceinline__ void umma_ts_warp(uint32_t tmem_d, uint32_t tmem_a, uint64_t bdesc, uint32_t idesc,
                                             uint32_t accumulate) {
    asm volatile(
        "{\n\t.reg .pred p, e;\n\t"
        "setp.ne.b32 p, %4, 0;\n\t"
        "elect.sync _|e, 0xffffffff;\n\t"
        "@e tcgen05.mma.cta_group::1.kind::f16 [%0], [%1], %2, %3, p;\n\t}" ::"r"(tmem_d),
        "r"(tmem_a), "l"(bdesc), "r"(idesc), "r"(accumulate)
        : "memory");
}
__device__ __forceinline__ void tmem_st8(uint32_t taddr, const uint32_t (&r)[8]) {
    asm volatile("tcgen05.st.sync.aligned.32x32b.x8.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};" ::"r"(taddr), "r"(r[0]),
                 "r"(r[1]), "r"(r[2]), "r"(r[3]), "r"(r[4]), "r"(r[5]), "r"(r[6]), "r"(r[7])
                 : "memory");
    asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
}

// A [128][32] fp16 (two K=16 steps), B [N][32] fp16, D [128][N] fp32
__global__ void __launch_bounds__(128, 1) k_ts(const __half *A, const __half *B, int N, float *D, int reps,
                                               long long *clk) {
    __shared__ __align__(1024) uint8_t bs[4 * 64 * 16];
    __shared__ uint64_t bar;
    __shared__ uint32_t slot;
    const int t = threadIdx.x, warp = t >> 5;
    // B: [chunk of 8 K][n][8]
    for (int i = t; i < N * 32; i += 128) {
        int n = i / 32, k = i % 32;
        reinterpret_cast<__half *>(bs)[((k / 8) * N + n) * 8 + (k % 8)] = B[n * 32 + k];
    }
    if (t == 0) { mbar_init(&bar, 1); fence_barrier_init(); }
    if (warp == 0) tmem_alloc(&slot, 256);
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tm = slot;
    // A row t -> lane t, columns 128.. (16 columns: K 0..31, two per column)
    uint32_t r[8];
    for (int s = 0; s < 2; s++) {
        for (int j = 0; j < 8; j++) {
            __half2 h = __halves2half2(A[t * 32 + s * 16 + 2 * j], A[t * 32 + s * 16 + 2 * j + 1]);
            r[j] = *reinterpret_cast<uint32_t *>(&h);
        }
        tmem_st8(tm + ((uint32_t)(warp * 32) << 16) + 128 + s * 8, r);
    }
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t idesc = umma_idesc_f16(128, N);
    const uint64_t bd = umma_desc(smem_u32(bs), N * 16, 128);
    long long t0 = clock64();
    if (warp == 0) {
        for (int s = 0; s < 2; s++) umma_ts_warp(tm, tm + 128 + s * 8, bd + ((s * 2 * N * 16) >> 4), idesc, s);
        for (int i = 0; i < reps; i++) umma_ts_warp(tm + 64 + (i & 1) * 32 * 0, tm + 128, bd, idesc, 1);
        umma_commit_warp(&bar);
    }
    mbar_wait(&bar, 0);
    long long t1 = clock64();
    tc_fence_after();
    uint32_t v[32];
    tmem_ld32(tm + ((uint32_t)(warp * 32) << 16), v);
    for (int n = 0; n < N && n < 32; n++) D[t * N + n] = __uint_as_float(v[n]);
    if (N > 32) {
        tmem_ld32(tm + ((uint32_t)(warp * 32) << 16) + 32, v);
        for (int n = 32; n < N; n++) D[t * N + n] = __uint_as_float(v[n - 32]);
    }
    if (t == 0) clk[0] = t1 - t0;
    tc_fence_before();
    __syncthreads();
    if (warp == 0) { tc_fence_after(); tmem_dealloc(tm, 256); }
}

int main() {
    for (int N : {32, 64}) {
        __half *A, *B; float *D; long long *clk;
        cudaMallocManaged(&A, 128 * 32 * 2); cudaMallocManaged(&B, 64 * 32 * 2);
        cudaMallocManaged(&D, 128 * 64 * 4); cudaMallocManaged(&clk, 8);
        float ha[128 * 32], hb[64 * 32];
        for (int i = 0; i < 128 * 32; i++) { ha[i] = (float)((i * 7 + 3) % 17 - 8); A[i] = __float2half(ha[i]); }
        for (int i = 0; i < N * 32; i++) { hb[i] = (float)((i * 5 + 1) % 13 - 6); B[i] = __float2half(hb[i]); }
        k_ts<<<1, 128>>>(A, B, N, D, 0, clk);
        cudaError_t e = cudaDeviceSynchronize();
        int bad = 0;
        for (int m = 0; m < 128; m++)
            for (int n = 0; n < N; n++) {
                float ref = 0;
                for (int k = 0; k < 32; k++) ref += ha[m * 32 + k] * hb[n * 32 + k];
                if (ref != D[m * N + n]) { if (bad < 4) printf("N=%d m=%d n=%d got %f want %f\n", N, m, n, D[m * N + n], ref); bad++; }
            }
        printf("TS layout N=%d: %s, %d mismatches\n", N, cudaGetErrorString(e), bad);
        const int reps = 4000;
        k_ts<<<148, 128>>>(A, B, N, D, reps, clk);
        e = cudaDeviceSynchronize();
        printf("TS rate N=%d: %.1f clk per MMA (%s)\n", N, (double)clk[0] / reps, cudaGetErrorString(e));
    }
    return 0;
}
