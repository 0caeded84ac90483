// jit.cpp -- PTX assembly (nvJitLink) + driver-API load/launch for the
// compiled path.  The paper compiles each SPN to a GPU binary through
// MLIR/NVVM/ptxas (§IV-C; compile times L415-416); here
// the generator emits PTX directly (codegen.cpp), so only the assembler runs.
#include "jit.h"

#include <cuda.h>
#include <dlfcn.h>

#include <mutex>
#include <unordered_map>

#include "spnb.h"

namespace spnb {

namespace {

// nvJitLink (PTX -> cubin; the toolkit's ptxas as a library), opened with dlopen
typedef void *NvjlHandle;
struct Nvjl {
    bool ok = false;
    std::string why;
    int (*create)(NvjlHandle *, uint32_t, const char **) = nullptr;
    int (*add)(NvjlHandle, int, const void *, size_t, const char *) = nullptr;
    int (*complete)(NvjlHandle) = nullptr;
    int (*cubin_size)(NvjlHandle, size_t *) = nullptr;
    int (*cubin)(NvjlHandle, void *) = nullptr;
    int (*log_size)(NvjlHandle, size_t *) = nullptr;
    int (*log)(NvjlHandle, char *) = nullptr;
    int (*destroy)(NvjlHandle *) = nullptr;
};

Nvjl &nvjl() {
    static Nvjl n;
    static std::once_flag once;
    std::call_once(once, [] {
        // the toolkit's copy first: a process may already hold an older
        // libnvJitLink.so.12 (e.g. one bundled with torch) under the soname
        const char *names[] = {"/usr/local/cuda/lib64/libnvJitLink.so.12",
                               "/usr/local/cuda/lib64/libnvJitLink.so", "libnvJitLink.so.12",
                               "libnvJitLink.so"};
        void *h = nullptr;
        for (const char *nm : names)
            if ((h = dlopen(nm, RTLD_NOW | RTLD_LOCAL))) break;
        if (!h) {
            n.why = "libnvJitLink.so not found";
            return;
        }
        // versioned entry points (the header's inline wrappers call these)
        const char *vers[] = {"_12_9", "_12_8", "_12_6", "_12_4", "_12_0"};
        for (const char *v : vers) {
            auto sym = [&](const char *base) { return dlsym(h, (std::string(base) + v).c_str()); };
            n.create = (decltype(n.create))sym("__nvJitLinkCreate");
            n.add = (decltype(n.add))sym("__nvJitLinkAddData");
            n.complete = (decltype(n.complete))sym("__nvJitLinkComplete");
            n.cubin_size = (decltype(n.cubin_size))sym("__nvJitLinkGetLinkedCubinSize");
            n.cubin = (decltype(n.cubin))sym("__nvJitLinkGetLinkedCubin");
            n.log_size = (decltype(n.log_size))sym("__nvJitLinkGetErrorLogSize");
            n.log = (decltype(n.log))sym("__nvJitLinkGetErrorLog");
            n.destroy = (decltype(n.destroy))sym("__nvJitLinkDestroy");
            n.ok = n.create && n.add && n.complete && n.cubin_size && n.cubin && n.log_size &&
                   n.log && n.destroy;
            if (n.ok) break;
        }
        if (!n.ok) n.why = "libnvJitLink.so lacks required symbols";
    });
    return n;
}

struct Driver {
    bool ok = false;
    std::string why;
    CUresult (*load)(CUmodule *, const void *) = nullptr;
    CUresult (*get_fn)(CUfunction *, CUmodule, const char *) = nullptr;
    CUresult (*launch)(CUfunction, unsigned, unsigned, unsigned, unsigned, unsigned, unsigned,
                       unsigned, CUstream, void **, void **) = nullptr;
    CUresult (*unload)(CUmodule) = nullptr;
    CUresult (*fn_attr)(int *, CUfunction_attribute, CUfunction) = nullptr;
    CUresult (*occ)(int *, CUfunction, int, size_t) = nullptr;
    CUresult (*err_str)(CUresult, const char **) = nullptr;
};

Driver &driver() {
    static Driver d;
    static std::once_flag once;
    std::call_once(once, [] {
        auto get = [&](const char *s, void **p) {
            cudaDriverEntryPointQueryResult q;
            return cudaGetDriverEntryPoint(s, p, cudaEnableDefault, &q) == cudaSuccess &&
                   q == cudaDriverEntryPointSuccess && *p;
        };
        d.ok = get("cuModuleLoadData", (void **)&d.load) &&
               get("cuModuleGetFunction", (void **)&d.get_fn) &&
               get("cuLaunchKernel", (void **)&d.launch) &&
               get("cuModuleUnload", (void **)&d.unload) &&
               get("cuFuncGetAttribute", (void **)&d.fn_attr) &&
               get("cuOccupancyMaxActiveBlocksPerMultiprocessor", (void **)&d.occ) &&
               get("cuGetErrorString", (void **)&d.err_str);
        if (!d.ok) d.why = "CUDA driver entry points unavailable";
    });
    return d;
}

std::string drv_msg(CUresult r, const char *where) {
    const char *s = nullptr;
    if (driver().err_str) driver().err_str(r, &s);
    return std::string(where) + ": " + (s ? s : "CUDA driver error");
}

std::mutex g_cache_mu;
std::unordered_map<std::string, std::vector<char>> g_cache;

}  // namespace

int jit_compile(const std::string &src, const std::string &arch, std::vector<char> &cubin,
                std::string &log) {
    const std::string key = arch + '\n' + src;
    {
        std::lock_guard<std::mutex> lk(g_cache_mu);
        auto it = g_cache.find(key);
        if (it != g_cache.end()) {
            cubin = it->second;
            return SPN_OK;
        }
    }
    Nvjl &n = nvjl();
    if (!n.ok) {
        log = n.why;
        return SPN_E_UNSUPPORTED;
    }
    // the generated PTX names its target; retarget it to this device's arch
    std::string ptx = src;
    const std::string tgt = ".target sm_100a";
    const size_t tp = ptx.find(tgt);
    if (tp != std::string::npos) ptx.replace(tp, tgt.size(), ".target sm_" + arch);
    const std::string a = "-arch=sm_" + arch;
    const char *opts[] = {a.c_str(), "-lineinfo"};
    NvjlHandle h = nullptr;
    if (n.create(&h, 2, opts) != 0) {
        log = "nvJitLinkCreate failed";
        return SPN_E_UNSUPPORTED;
    }
    int r = n.add(h, 2 /* NVJITLINK_INPUT_PTX */, ptx.data(), ptx.size(), "spnb_task.ptx");
    if (r == 0) r = n.complete(h);
    if (r != 0) {
        size_t ls = 0;
        n.log_size(h, &ls);
        std::string l(ls, '\0');
        if (ls) n.log(h, &l[0]);
        n.destroy(&h);
        log = "nvJitLink: " + l;
        return SPN_E_UNSUPPORTED;
    }
    size_t cs = 0;
    n.cubin_size(h, &cs);
    cubin.assign(cs, 0);
    n.cubin(h, cubin.data());
    n.destroy(&h);
    std::lock_guard<std::mutex> lk(g_cache_mu);
    g_cache[key] = cubin;
    return SPN_OK;
}

int jit_load(const std::vector<char> &cubin, const std::string &name, int v, int block,
             JitKernel &k, std::string &msg) {
    Driver &d = driver();
    if (!d.ok) {
        msg = d.why;
        return SPN_E_CUDA;
    }
    cudaFree(nullptr);  // make the runtime's primary context current
    CUmodule m;
    CUresult r = d.load(&m, cubin.data());
    if (r != CUDA_SUCCESS) {
        msg = drv_msg(r, "cuModuleLoadData");
        return SPN_E_CUDA;
    }
    k.module[v] = m;
    CUfunction f;
    const std::string fn = name + (v ? "_m" : "_j");
    if ((r = d.get_fn(&f, m, fn.c_str())) != CUDA_SUCCESS) {
        msg = drv_msg(r, "cuModuleGetFunction");
        return SPN_E_CUDA;
    }
    k.fn[v] = f;
    d.fn_attr(&k.regs[v], CU_FUNC_ATTRIBUTE_NUM_REGS, f);
    d.fn_attr(&k.local_bytes[v], CU_FUNC_ATTRIBUTE_LOCAL_SIZE_BYTES, f);
    d.occ(&k.occupancy[v], f, block, 0);
    k.block[v] = block;
    return SPN_OK;
}

int jit_launch(const JitKernel &k, bool marg, int grid, int block, cudaStream_t st,
               const float *x, long long n, long long ld, float *out, int R, int *argmax,
               const float *tab, std::string &msg) {
    Driver &d = driver();
    void *args[] = {(void *)&x, (void *)&n, (void *)&ld, (void *)&out, (void *)&R, (void *)&argmax,
                    (void *)&tab};
    const CUresult r = d.launch((CUfunction)k.fn[marg ? 1 : 0], (unsigned)grid, 1, 1,
                                (unsigned)block, 1, 1, 0, (CUstream)st, args, nullptr);
    if (r != CUDA_SUCCESS) {
        msg = drv_msg(r, "cuLaunchKernel");
        return SPN_E_CUDA;
    }
    return SPN_OK;
}

void jit_unload_variant(JitKernel &k, int v) {
    if (k.module[v] && driver().ok) driver().unload((CUmodule)k.module[v]);
    k.module[v] = nullptr;
    k.fn[v] = nullptr;
}

void jit_unload(JitKernel &k) {
    for (int v = 0; v < 2; ++v) jit_unload_variant(k, v);
}

}  // namespace spnb
