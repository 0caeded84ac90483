// FP32 FMA issue-rate microbenchmark on sm_100a: 3-register FFMA, immediate
// FFMA, packed FFMA2 (fma.rn.f32x2).  Prints lane-FMA/clk/SM for each.
#include <cstdio>
#include <cuda_runtime.h>
#define N_IT 4096
__global__ void k_reg(float *o, float a, float b) {
    float x[8];
    for (int i = 0; i < 8; ++i) x[i] = threadIdx.x + i;
    float y = a * threadIdx.x, z = b * threadIdx.x;
    for (int it = 0; it < N_IT; ++it)
#pragma unroll
        for (int i = 0; i < 8; ++i) asm volatile("fma.rn.f32 %0, %0, %1, %2;" : "+f"(x[i]) : "f"(y), "f"(z));
    float s = 0; for (int i = 0; i < 8; ++i) s += x[i];
    o[blockIdx.x * blockDim.x + threadIdx.x] = s;
}
__global__ void k_imm(float *o, float a, float b) {
    float x[8];
    for (int i = 0; i < 8; ++i) x[i] = threadIdx.x + i;
    for (int it = 0; it < N_IT; ++it)
#pragma unroll
        for (int i = 0; i < 8; ++i) asm volatile("fma.rn.f32 %0, %0, 0f3F7FBE77, 0f3F000000;" : "+f"(x[i]));
    float s = 0; for (int i = 0; i < 8; ++i) s += x[i];
    o[blockIdx.x * blockDim.x + threadIdx.x] = s;
}
__global__ void k_imm_b(float *o, float a, float b) {  // imm multiplier, register addend
    float x[8];
    for (int i = 0; i < 8; ++i) x[i] = threadIdx.x + i;
    float z = b * threadIdx.x;
    for (int it = 0; it < N_IT; ++it)
#pragma unroll
        for (int i = 0; i < 8; ++i) asm volatile("fma.rn.f32 %0, %0, 0f3F7FBE77, %1;" : "+f"(x[i]) : "f"(z));
    float s = 0; for (int i = 0; i < 8; ++i) s += x[i];
    o[blockIdx.x * blockDim.x + threadIdx.x] = s;
}
__global__ void k_ffma2(float *o, float a, float b) {
    unsigned long long x[4], y, z;
    for (int i = 0; i < 4; ++i) {
        float u = threadIdx.x + i, v = u + 1;
        asm("mov.b64 %0, {%1,%2};" : "=l"(x[i]) : "f"(u), "f"(v));
    }
    { float u = a * threadIdx.x; asm("mov.b64 %0, {%1,%1};" : "=l"(y) : "f"(u)); }
    { float u = b * threadIdx.x; asm("mov.b64 %0, {%1,%1};" : "=l"(z) : "f"(u)); }
    for (int it = 0; it < N_IT; ++it)
#pragma unroll
        for (int i = 0; i < 4; ++i) asm volatile("fma.rn.f32x2 %0, %0, %1, %2;" : "+l"(x[i]) : "l"(y), "l"(z));
    float s = 0;
    for (int i = 0; i < 4; ++i) { float u, v; asm("mov.b64 {%0,%1}, %2;" : "=f"(u), "=f"(v) : "l"(x[i])); s += u + v; }
    o[blockIdx.x * blockDim.x + threadIdx.x] = s;
}
int main() {
    int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    int clk; cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
    float *o; cudaMalloc(&o, 1 << 26);
    const int blocks = sms * 4, threads = 512;
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
    const char *names[] = {"ffma_3reg", "ffma_imm_imm", "ffma_imm_reg", "ffma2_f32x2"};
    void (*ks[])(float *, float, float) = {k_reg, k_imm, k_imm_b, k_ffma2};
    for (int v = 0; v < 4; ++v) {
        for (int rep = 0; rep < 2; ++rep) {
            cudaEventRecord(e0);
            ks[v]<<<blocks, threads>>>(o, 1.0001f, 0.5f);
            cudaEventRecord(e1); cudaEventSynchronize(e1);
        }
        float ms; cudaEventElapsedTime(&ms, e0, e1);
        double fmas = (double)blocks * threads * N_IT * 8;
        printf("%-14s %.3f ms  %.1f lane-FMA/clk/SM (at %d MHz nominal)  %.2f TFMA/s\n", names[v], ms,
               fmas / (ms * 1e-3) / sms / (clk * 1e3), clk / 1000, fmas / (ms * 1e-3) / 1e12);
    }
    return 0;
}
