// argmax.cu -- per-sample argmax over the roots (class decision of the
// speaker-identification application), for compiled plans whose
// roots are spread over several generated kernels (otherwise the argmax is
// fused into the generated kernel).  Reading c10: the lowest index among the
// largest non-NaN values; -1 if every root is NaN.
#include <cuda_runtime.h>
#include <math_constants.h>
#include <stdint.h>

namespace spnb {

__global__ void argmax_rows_kernel(const float *__restrict__ out, int64_t n, int R,
                                   int32_t *__restrict__ argmax) {
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t s = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; s < n; s += stride) {
        const float *o = out + s * R;
        float best = -CUDART_INF_F;
        int idx = -1;
        for (int r = 0; r < R; ++r) {
            const float w = __ldg(o + r);
            if (!(w != w) && (idx < 0 || w > best)) {
                best = w;
                idx = r;
            }
        }
        argmax[s] = idx;
    }
}

cudaError_t argmax_rows_launch(const float *out, int64_t n, int R, int32_t *argmax,
                               cudaStream_t st) {
    if (n <= 0) return cudaSuccess;
    int dev = 0, sms = 148;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    const int64_t need = (n + 255) / 256;
    const int grid = (int)(need < (int64_t)sms * 8 ? need : (int64_t)sms * 8);
    argmax_rows_kernel<<<grid, 256, 0, st>>>(out, n, R, argmax);
    return cudaGetLastError();
}

}  // namespace spnb
