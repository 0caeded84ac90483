// tcgen05.mma kind::f16 throughput with K-major SWIZZLE_NONE shared-memory
// operands (the layered kernel's layout): M=128, N in {240, 256}, K=48 per
// group (3 MMAs of K=16); thread 0 issues ITERS groups back to back, one
// commit + wait at the end.  Prints dense flop/clk/SM.
#include <cstdint>
#include <cstdio>
#include <cuda_runtime.h>
#define ITERS 512
__device__ __forceinline__ uint64_t desc(uint32_t addr, uint32_t lbo, uint32_t sbo) {
    uint64_t d = 0;
    d |= (uint64_t)((addr >> 4) & 0x3FFFu);
    d |= (uint64_t)((lbo >> 4) & 0x3FFFu) << 16;
    d |= (uint64_t)((sbo >> 4) & 0x3FFFu) << 32;
    d |= (uint64_t)1 << 46;
    return d;
}
__global__ void k(int N, int kpad, int nacc, unsigned long long *cyc) {
    extern __shared__ __align__(1024) uint8_t sm[];
    __shared__ uint32_t slot;
    __shared__ __align__(8) uint64_t bar;
    const int RT = 128;
    for (int i = threadIdx.x; i < (RT + 256) * kpad * 2 / 4; i += blockDim.x) ((uint32_t *)sm)[i] = 0x3c003c00u;
    if (threadIdx.x < 32) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"((uint32_t)__cvta_generic_to_shared(&slot)));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    if (threadIdx.x == 0) {
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"((uint32_t)__cvta_generic_to_shared(&bar)));
        asm volatile("fence.mbarrier_init.release.cluster;");
    }
    asm volatile("fence.proxy.async.shared::cta;");
    asm volatile("tcgen05.fence::before_thread_sync;");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;");
    if (threadIdx.x == 0) {
        const uint32_t a = (uint32_t)__cvta_generic_to_shared(sm), b = a + RT * kpad * 2;
        const uint32_t lbo_a = RT * 16, lbo_b = N * 16;
        const uint32_t idesc = (1u << 4) | ((uint32_t)(N >> 3) << 17) | ((uint32_t)(RT >> 4) << 24);
        const unsigned long long t0 = clock64();
        for (int it = 0; it < ITERS; it += nacc)
            for (int kk = 0; kk < kpad / 16; ++kk)
                for (int q = 0; q < nacc; ++q) {  // nacc independent accumulators, interleaved
                    const uint64_t da = desc(a + kk * 2 * lbo_a, lbo_a, 128), db = desc(b + kk * 2 * lbo_b, lbo_b, 128);
                    const uint32_t acc = kk > 0;
                    asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                                 "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}\n" ::"r"(slot + q * 128),
                                 "l"(da), "l"(db), "r"(idesc), "r"(acc));
                }
        asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"((uint32_t)__cvta_generic_to_shared(&bar)));
        uint32_t done = 0;
        while (!done)
            asm volatile("{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], 0;\n\tselp.u32 %0, 1, 0, p;\n\t}\n"
                         : "=r"(done) : "r"((uint32_t)__cvta_generic_to_shared(&bar)));
        cyc[blockIdx.x] = clock64() - t0;
    }
    asm volatile("tcgen05.fence::before_thread_sync;");
    __syncthreads();
    if (threadIdx.x < 32) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(slot));
}
int main() {
    int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    unsigned long long *c; cudaMalloc(&c, 8 * 1024);
    cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
    for (int nacc : {1, 2, 4}) for (int N : {240, 120}) for (int kp : {48}) {
        if (nacc * N > 512 || (nacc > 1 && N > 128)) continue;
        k<<<sms, 128, (128 + 256) * kp * 2>>>(N, kp, nacc, c);
        cudaError_t e = cudaDeviceSynchronize();
        unsigned long long h; cudaMemcpy(&h, c, 8, cudaMemcpyDeviceToHost);
        const double flop = 2.0 * 128 * N * kp * ITERS;
        printf("M=128 N=%3d K=%d accumulators=%d (noswizzle): %.0f flop/clk/SM (%llu clk) %s\n", N, kp, nacc, flop / h, h, cudaGetErrorString(e));
    }
    return 0;
}
