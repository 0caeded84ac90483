// TMEM read-throughput microbenchmark on sm_100a: tcgen05.ld.32x32b.x{8,16,32}
// issued by W warps of one CTA per SM (warp w reads lane quarter w%4).
// Prints bytes/clk/SM.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
#define ITERS 2048
template <int X>
__device__ __forceinline__ void ld(uint32_t a, float *v);
template <> __device__ __forceinline__ void ld<8>(uint32_t a, float *v) {
    asm volatile("tcgen05.ld.sync.aligned.32x32b.x8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                 : "=f"(v[0]), "=f"(v[1]), "=f"(v[2]), "=f"(v[3]), "=f"(v[4]), "=f"(v[5]), "=f"(v[6]), "=f"(v[7]) : "r"(a));
}
template <> __device__ __forceinline__ void ld<16>(uint32_t a, float *v) {
    asm volatile("tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
                 : "=f"(v[0]), "=f"(v[1]), "=f"(v[2]), "=f"(v[3]), "=f"(v[4]), "=f"(v[5]), "=f"(v[6]), "=f"(v[7]),
                   "=f"(v[8]), "=f"(v[9]), "=f"(v[10]), "=f"(v[11]), "=f"(v[12]), "=f"(v[13]), "=f"(v[14]), "=f"(v[15]) : "r"(a));
}
template <int X>
__global__ void k(float *out, unsigned long long *cyc) {
    __shared__ uint32_t slot;
    const int warp = threadIdx.x >> 5;
    if (warp == 0) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"((uint32_t)__cvta_generic_to_shared(&slot)));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    asm volatile("tcgen05.fence::before_thread_sync;");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;");
    const uint32_t tm = slot + ((uint32_t)((warp & 3) * 32) << 16);
    float acc = 0.f;
    const unsigned long long t0 = clock64();
    for (int it = 0; it < ITERS; ++it) {
        float v[4][X];
#pragma unroll
        for (int b = 0; b < 4; ++b) ld<X>(tm + ((it * 4 + b) * X) % 512, v[b]);
        asm volatile("tcgen05.wait::ld.sync.aligned;");
#pragma unroll
        for (int b = 0; b < 4; ++b)
#pragma unroll
            for (int i = 0; i < X; ++i) acc += v[b][i];
    }
    const unsigned long long t1 = clock64();
    asm volatile("tcgen05.fence::before_thread_sync;");
    __syncthreads();
    if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(slot));
    out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
    if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
}
template <int X>
void run(int sms, int warps, float *o, unsigned long long *c) {
    k<X><<<sms, warps * 32>>>(o, c);
    cudaDeviceSynchronize();
    unsigned long long h;
    cudaMemcpy(&h, c, 8, cudaMemcpyDeviceToHost);
    const double bytes = (double)warps * 32 * 4 * X * 4 * ITERS;
    printf("32x32b.x%-2d warps %2d: %.1f B/clk/SM (%llu clk)  err=%s\n", X, warps, bytes / h, h,
           cudaGetErrorString(cudaGetLastError()));
}
int main() {
    int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    float *o; unsigned long long *c;
    cudaMalloc(&o, 1 << 24); cudaMalloc(&c, 8 * 1024);
    for (int w : {4, 8, 16}) { run<8>(sms, w, o, c); run<16>(sms, w, o, c); }
    return 0;
}
