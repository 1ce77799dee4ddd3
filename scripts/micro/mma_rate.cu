// Microbenchmark: tcgen05.mma (kind::f16, SS operands, no-swizzle K-major) issue rate
// from one thread vs N, and the cost of a commit + wait round trip.
#include <cstdio>
#include <cuda_runtime.h>
#include "../../paper_conf_sigmod_bastanim22_b200/csrc/common.cuh"
using namespace otif;

__device__ __forceinline__ void umma_elect(uint32_t tmem_d, uint64_t adesc, uint64_t bdesc, uint32_t idesc,
                                           uint32_t accumulate) {
    asm volatile(
        "{\n\t.reg .pred p, e;\n\t"
        "setp.ne.b32 p, %4, 0;\n\t"
        "elect.sync _|e, 0xffffffff;\n\t"
        "@e tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(tmem_d),
        "l"(adesc), "l"(bdesc), "r"(idesc), "r"(accumulate)
        : "memory");
}
__device__ __forceinline__ void commit_elect(uint64_t *bar) {
    asm volatile("{\n\t.reg .pred e;\n\telect.sync _|e, 0xffffffff;\n\t"
                 "@e tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];\n\t}" ::"r"(smem_u32(bar))
                 : "memory");
}
__global__ void __launch_bounds__(128, 1) k_rate(int N, int reps, int mode, long long *out) {
    __shared__ __align__(1024) uint8_t sm[4 * 128 * 16 + 4 * 256 * 16];
    __shared__ uint64_t bar;
    __shared__ uint32_t slot;
    for (int i = threadIdx.x; i < (int)sizeof(sm) / 4; i += blockDim.x) reinterpret_cast<uint32_t *>(sm)[i] = 0;
    if (threadIdx.x == 0) { mbar_init(&bar, 1); fence_barrier_init(); }
    if (threadIdx.x < 32) tmem_alloc(&slot, 512);
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem = slot;
    if (mode >= 3 && threadIdx.x < 32) {
        const uint32_t a = smem_u32(sm), b = a + 4 * 128 * 16;
        const uint32_t idesc = umma_idesc_bf16(128, N);
        uint32_t ph = 0;
        long long t0 = clock64();
        if (mode == 3) {
            for (int r = 0; r < reps; r++) {
                const uint32_t sh = (r * 7) & 15;
                umma_elect(tmem + (r & 1) * 256, umma_desc(a + sh * 16, 2048, 128), umma_desc(b + (r & 1) * 1024, N * 16, 128),
                           idesc, 1);
            }
        } else {
            const uint64_t ad0 = umma_desc(a, 2048, 128), bd0 = umma_desc(b, N * 16, 128);
            for (int r = 0; r < reps; r++) {
                const uint32_t sh = (r * 7) & 15;
                umma_elect(tmem + (r & 1) * 256, ad0 + sh, bd0 + (r & 1) * 64, idesc, 1);
            }
        }
        commit_elect(&bar);
        mbar_wait(&bar, ph);
        long long t1 = clock64();
        if (blockIdx.x == 0 && threadIdx.x == 0) out[0] = t1 - t0;
    }
    if (mode < 3 && threadIdx.x == 0) {
        const uint32_t a = smem_u32(sm), b = a + 4 * 128 * 16;
        const uint32_t idesc = umma_idesc_bf16(128, N);
        const uint64_t ad = umma_desc(a, 2048, 128), bd = umma_desc(b, N * 16, 128);
        uint32_t ph = 0;
        // warm
        umma_bf16(tmem, ad, bd, idesc, 0);
        umma_commit(&bar);
        mbar_wait(&bar, ph); ph ^= 1;
        long long t0 = clock64();
        if (mode == 0) {
            for (int r = 0; r < reps; r++) umma_bf16(tmem, ad, bd, idesc, 1);
            umma_commit(&bar);
            mbar_wait(&bar, ph); ph ^= 1;
        } else if (mode == 1) {  // commit + wait after every MMA (round-trip latency)
            for (int r = 0; r < reps; r++) {
                umma_bf16(tmem, ad, bd, idesc, 1);
                umma_commit(&bar);
                mbar_wait(&bar, ph); ph ^= 1;
            }
        } else {  // descriptors recomputed per MMA from loop state (like a real loop)
            for (int r = 0; r < reps; r++) {
                const uint32_t sh = (r * 7) & 15;
                umma_bf16(tmem + (r & 1) * 256, umma_desc(a + sh * 16, 2048, 128), umma_desc(b + (r & 1) * 1024, N * 16, 128),
                          idesc, 1);
            }
            umma_commit(&bar);
            mbar_wait(&bar, ph); ph ^= 1;
        }
        long long t1 = clock64();
        if (blockIdx.x == 0) out[0] = t1 - t0;
    }
    tc_fence_before();
    __syncthreads();
    if (threadIdx.x < 32) { tc_fence_after(); tmem_dealloc(tmem, 512); }
}

int main() {
    long long *d;
    cudaMalloc(&d, 8);
    for (int mode = 0; mode < 5; mode++)
        for (int N : {32, 64, 128, 256}) {
            const int reps = mode == 1 ? 200 : 4000;
            k_rate<<<148, 128>>>(N, reps, mode, d);
            cudaError_t e = cudaDeviceSynchronize();
            long long h = 0;
            cudaMemcpy(&h, d, 8, cudaMemcpyDeviceToHost);
            printf("mode %d N %3d: %.1f clk per MMA (%s)  floor %d\n", mode, N, (double)h / reps, cudaGetErrorString(e), 128 * N / 256);
        }
    return 0;
}
