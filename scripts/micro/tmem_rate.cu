// Microbenchmark: tcgen05.ld (32x32b.x32) throughput vs warps, and the cost of
// fence.proxy.async.shared::cta after shared-memory stores.
#include <cstdio>
#include <cuda_runtime.h>
#include "../../paper_conf_sigmod_bastanim22_b200/csrc/common.cuh"
using namespace otif;

__global__ void __launch_bounds__(512, 1) k_ld(int nwarps, int reps, long long *out) {
    __shared__ uint32_t slot;
    __shared__ __align__(16) uint8_t sm[512 * 64];
    const int warp = threadIdx.x >> 5;
    if (warp == 0) tmem_alloc(&slot, 512);
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem = slot;
    uint32_t acc = 0;
    long long t0 = clock64();
    if (warp < nwarps) {
        for (int r = 0; r < reps; r++) {
            uint32_t v[32];
            tmem_ld32(tmem + ((uint32_t)((warp & 3) * 32) << 16) + ((r * 32 + (warp >> 2) * 64) & 511), v);
#pragma unroll
            for (int j = 0; j < 32; j++) acc += v[j];
        }
    }
    __syncthreads();
    long long t1 = clock64();
    if (threadIdx.x == 0 && blockIdx.x == 0) out[0] = t1 - t0;
    // fence cost: each thread stores 64 B then fences
    long long t2 = clock64();
    if (warp < nwarps) {
        for (int r = 0; r < reps; r++) {
            *reinterpret_cast<uint4 *>(sm + threadIdx.x * 64) = make_uint4(acc, r, 0, 0);
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        }
    }
    __syncthreads();
    long long t3 = clock64();
    if (threadIdx.x == 0 && blockIdx.x == 0) out[1] = t3 - t2;
    if (acc == 0x12345678) out[2] = acc;
    tc_fence_before();
    __syncthreads();
    if (warp == 0) { tc_fence_after(); tmem_dealloc(tmem, 512); }
}

int main() {
    long long *d;
    cudaMalloc(&d, 24);
    for (int nw : {1, 4, 8, 16}) {
        const int reps = 1000;
        k_ld<<<148, 512>>>(nw, reps, d);
        cudaError_t e = cudaDeviceSynchronize();
        long long h[2];
        cudaMemcpy(h, d, 16, cudaMemcpyDeviceToHost);
        printf("warps %2d: tcgen05.ld x32: %.1f clk per warp-load (%.1f B/clk per SM); fence.proxy.async: %.1f clk per iter (%s)\n",
               nw, (double)h[0] / reps, (double)nw * 4096 * reps / h[0], (double)h[1] / reps, cudaGetErrorString(e));
    }
    return 0;
}
