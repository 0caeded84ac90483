// tcgen05.mma issue cost in the layered v2 kernel's pattern: batches of
// nacc groups x 3 K-steps (M=128, N, K=16 each, f16, K-major SWIZZLE_NONE
// operands in shared memory), K-steps interleaved across the batch, then
// `commits` tcgen05.commit per batch; optionally 4 more warps stream
// tcgen05.ld from other TMEM columns (the epilogue's reads).  Thread 0 of
// warp 4 issues; prints clk per MMA and flop/clk/SM.
// build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o umma_issue umma_issue.cu
#include <cstdint>
#include <cstdio>
#include <cuda_runtime.h>
#define BATCHES 256
__device__ __forceinline__ uint64_t desc(uint32_t addr, uint32_t lbo, uint32_t sbo) {
    uint64_t d = 0;
    d |= (uint64_t)((addr >> 4) & 0x3FFFu);
    d |= (uint64_t)((lbo >> 4) & 0x3FFFu) << 16;
    d |= (uint64_t)((sbo >> 4) & 0x3FFFu) << 32;
    d |= (uint64_t)1 << 46;
    return d;
}
__global__ void k(int N, int nacc, int commits, int readers, unsigned long long *cyc, int seq) {
    extern __shared__ __align__(1024) uint8_t sm[];
    __shared__ uint32_t slot;
    __shared__ __align__(8) uint64_t bar[16];
    __shared__ volatile int stop;
    const int RT = 128, kpad = 48;
    const int warp = threadIdx.x >> 5;
    for (int i = threadIdx.x; i < (RT + 4 * 256) * kpad * 2 / 4; i += blockDim.x) ((uint32_t *)sm)[i] = 0x3c003c00u;
    if (warp == 4) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"((uint32_t)__cvta_generic_to_shared(&slot)));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    if (threadIdx.x == 0) {
        stop = 0;
        for (int i = 0; i < 16; ++i)
            asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"((uint32_t)__cvta_generic_to_shared(&bar[i])));
        asm volatile("fence.mbarrier_init.release.cluster;");
    }
    asm volatile("fence.proxy.async.shared::cta;");
    asm volatile("tcgen05.fence::before_thread_sync;");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;");
    const uint32_t tmem = slot;
    if (warp == 4 && (threadIdx.x & 31) == 0) {
        const uint32_t a = (uint32_t)__cvta_generic_to_shared(sm);
        const uint32_t lbo_a = RT * 16, lbo_b = N * 16;
        const uint32_t idesc = (1u << 4) | ((uint32_t)(N >> 3) << 17) | ((uint32_t)(RT >> 4) << 24);
        const unsigned long long t0 = clock64();
        for (int it = 0; it < BATCHES; ++it) {
            for (int kq = 0; kq < (kpad / 16) * nacc; ++kq) {
                // seq = 0: K-steps interleaved across the nacc accumulators;
                // seq = 1: each accumulator's K-steps back to back (groups in turn)
                const int kk = seq ? kq % (kpad / 16) : kq / nacc, q = seq ? kq / (kpad / 16) : kq % nacc;
                {
                    const uint32_t b = a + RT * kpad * 2 + q * 256 * kpad * 2;
                    const uint64_t da = desc(a + kk * 2 * lbo_a, lbo_a, 128), db = desc(b + kk * 2 * lbo_b, lbo_b, 128);
                    asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                                 "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}\n" ::"r"(tmem + q * N),
                                 "l"(da), "l"(db), "r"(idesc), "r"((uint32_t)(kk > 0)));
                }
            }
            for (int c = 0; c < commits; ++c)
                asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(
                    (uint32_t)__cvta_generic_to_shared(&bar[c])));
        }
        asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"((uint32_t)__cvta_generic_to_shared(&bar[15])));
        uint32_t done = 0;
        while (!done)
            asm volatile("{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], 0;\n\tselp.u32 %0, 1, 0, p;\n\t}\n"
                         : "=r"(done) : "r"((uint32_t)__cvta_generic_to_shared(&bar[15])));
        cyc[blockIdx.x] = clock64() - t0;
        stop = 1;
    }
    if (warp < 4 && readers) {
        // epilogue-like TMEM reads of columns 400..479 until the issuer is done
        const uint32_t base = tmem + ((uint32_t)(warp * 32) << 16) + 400;
        float acc = 0.f;
        while (!stop) {
            uint32_t r[16];
            asm volatile("tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
                         : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
                           "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15])
                         : "r"(base));
            asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
            for (int j = 0; j < 16; ++j) acc += __uint_as_float(r[j]);
        }
        if (acc == 12345.f) cyc[1023] = 1;
    }
    asm volatile("tcgen05.fence::before_thread_sync;");
    __syncthreads();
    if (warp == 4) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(tmem));
}
int main() {
    int sms;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    unsigned long long *c;
    cudaMalloc(&c, 8 * 1024);
    cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
    const size_t smem = (128 + 4 * 256) * 48 * 2;
    for (int seq : {0, 1})
    for (int readers : {0, 1})
        for (int N : {80, 96, 128, 160, 240, 256})
            for (int nacc : {1, 2, 3, 4})
                for (int commits : {1}) {
                    if (nacc * N > 512 || (seq && nacc == 1)) continue;
                    k<<<sms, 160, smem>>>(N, nacc, commits, readers, c, seq);
                    cudaError_t e = cudaDeviceSynchronize();
                    unsigned long long h;
                    cudaMemcpy(&h, c, 8, cudaMemcpyDeviceToHost);
                    const double mmas = (double)BATCHES * nacc * 3;
                    const double flop = mmas * 2.0 * 128 * N * 16;
                    printf("seq=%d readers=%d N=%3d acc=%d commits/batch=%d: %6.1f clk/MMA %6.0f flop/clk/SM %s\n", seq, readers, N,
                           nacc, commits, h / mmas, flop / h, cudaGetErrorString(e));
                }
    return 0;
}
