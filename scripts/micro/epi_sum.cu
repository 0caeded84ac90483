// Cost of the layered v2 epilogue's per-sum sequence in isolation: 4 warps
// (one per TMEM lane quarter), per sum: tcgen05.ld of 2 x 20 columns
// (double-buffered halves), 20 FFMA2 against 40 registers of ea, lg2,
// subtract a per-sum constant (LDG), tcgen05.st of the result into another
// column.  Variants drop parts to attribute the cycles.
// build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o epi_sum epi_sum.cu
#include <cstdint>
#include <cstdio>
#include <cuda_runtime.h>
#define NSUM 4096
__device__ __forceinline__ void ld8(uint32_t a, float *v) {
    uint32_t r[8];
    asm volatile("tcgen05.ld.sync.aligned.32x32b.x8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                 : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7])
                 : "r"(a));
    for (int k = 0; k < 8; ++k) v[k] = __uint_as_float(r[k]);
}
__device__ __forceinline__ void ld4(uint32_t a, float *v) {
    uint32_t r[4];
    asm volatile("tcgen05.ld.sync.aligned.32x32b.x4.b32 {%0,%1,%2,%3}, [%4];"
                 : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]) : "r"(a));
    for (int k = 0; k < 4; ++k) v[k] = __uint_as_float(r[k]);
}
__device__ __forceinline__ void ld20(uint32_t a, float (&t)[20]) { ld8(a, t); ld8(a + 8, t + 8); ld4(a + 16, t + 16); }
__device__ __forceinline__ void waitld() { asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory"); }
__device__ __forceinline__ float dot(const float *e, const float (&t)[20]) {
    float2 p0 = make_float2(0.f, 0.f), p1 = make_float2(0.f, 0.f);
#pragma unroll
    for (int i = 0; i < 20; i += 4) {
        p0 = __ffma2_rn(make_float2(e[i], e[i + 1]), make_float2(t[i], t[i + 1]), p0);
        p1 = __ffma2_rn(make_float2(e[i + 2], e[i + 3]), make_float2(t[i + 2], t[i + 3]), p1);
    }
    return (p0.x + p0.y) + (p1.x + p1.y);
}
template <int VAR>
__global__ void k(const float *ks, float *sink, unsigned long long *cyc) {
    __shared__ uint32_t slot;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (warp == 0) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"((uint32_t)__cvta_generic_to_shared(&slot)));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    asm volatile("tcgen05.fence::before_thread_sync;");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;");
    const uint32_t base = slot + ((uint32_t)(warp * 32) << 16);
    float ear[40];
    for (int i = 0; i < 40; ++i) ear[i] = 1.f / (i + 1 + lane);
    float b0[20], b1[20];
    float acc_all = 0.f;
    const unsigned long long t0 = clock64();
    ld20(base, b0);
    waitld();
    for (int s = 0; s < NSUM; ++s) {
        const uint32_t row = base + (uint32_t)((s % 4) * 40);
        ld20(row + 20, b1);
        float a = dot(ear, b0);
        if (VAR != 1) waitld();
        ld20(row + 40, b0);
        a += dot(ear + 20, b1);
        float val = (VAR == 2) ? a : (__logf(a) * 1.4427f);
        if (VAR != 3) val -= __ldg(ks + (s & 63));
        if (VAR == 0 || VAR == 1 || VAR == 2 || VAR == 3)
            asm volatile("tcgen05.st.sync.aligned.32x32b.x1.b32 [%0], {%1};" ::"r"(base + 400 + (s & 63)), "r"(__float_as_uint(val)));
        else
            acc_all += val;
        waitld();
    }
    asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
    const unsigned long long t1 = clock64();
    if (lane == 0) cyc[blockIdx.x * 4 + warp] = t1 - t0;
    sink[threadIdx.x] = acc_all + b0[0];
    asm volatile("tcgen05.fence::before_thread_sync;");
    __syncthreads();
    if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(slot));
}
int main() {
    float *ks, *sink;
    unsigned long long *c;
    cudaMalloc(&ks, 4096);
    cudaMemset(ks, 0, 4096);
    cudaMalloc(&sink, 4096);
    cudaMalloc(&c, 8 * 1024);
    const char *names[] = {"full (ld/wait/ffma2/lg2/ldg/st)", "no mid wait (one wait per sum)", "no lg2",
                           "no ldg", "no tcgen05.st"};
    void (*fns[])(const float *, float *, unsigned long long *) = {k<0>, k<1>, k<2>, k<3>, k<4>};
    for (int v = 0; v < 5; ++v) {
        fns[v]<<<1, 128>>>(ks, sink, c);
        cudaError_t e = cudaDeviceSynchronize();
        unsigned long long h[4];
        cudaMemcpy(h, c, sizeof(h), cudaMemcpyDeviceToHost);
        printf("%-36s %7.1f clk/sum (warp0) %s\n", names[v], (double)h[0] / NSUM, cudaGetErrorString(e));
    }
    return 0;
}
