// jit.h -- PTX assembly and driver-API loading of the compiled path's
// generated kernels (codegen.h).  nvJitLink is opened with dlopen and the
// driver entry points are obtained through the runtime
// (cudaGetDriverEntryPoint), so libspnb.so loads (and can generate and
// assemble kernels) without a GPU.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include <string>
#include <vector>

namespace spnb {

// Assemble generated PTX to a cubin for sm_<arch> (e.g. "100a").  Results
// are cached in-process by source text.  Returns SPN_OK, or
// SPN_E_UNSUPPORTED (nvJitLink missing or an assembler error; log says why).
int jit_compile(const std::string &src, const std::string &arch, std::vector<char> &cubin,
                std::string &log);

struct JitKernel {
    void *module[2] = {nullptr, nullptr};  // CUmodule per variant
    void *fn[2] = {nullptr, nullptr};      // CUfunction: [0] joint, [1] marginal
    int regs[2] = {0, 0};
    int occupancy[2] = {0, 0};  // CTAs per SM at the launch block size
    int local_bytes[2] = {0, 0};  // per-thread local memory (> 0: register spills)
    int block[2] = {0, 0};        // threads per CTA the variant was generated for
};

// Load variant v's cubin (0 joint, 1 marginal) into the current context and
// look up its entry <name>_j / <name>_m.
int jit_load(const std::vector<char> &cubin, const std::string &name, int v, int block,
             JitKernel &k, std::string &msg);
// Launch with (x, n, ld, out, R, argmax, tab) arguments.
int jit_launch(const JitKernel &k, bool marg, int grid, int block, cudaStream_t st,
               const float *x, long long n, long long ld, float *out, int R, int *argmax,
               const float *tab, std::string &msg);
void jit_unload(JitKernel &k);
void jit_unload_variant(JitKernel &k, int v);  // one of the two modules

}  // namespace spnb
