// codegen.h -- per-SPN code generation for the compiled path (kernel KS).
//
// The paper compiles every SPN to its own GPU kernel (§IV-C,
// L369-382: one thread per sample, the DAG as straight-line code, constants
// folded in).  This generator does the same for sm_100a from the canonical
// DAG: every inner node becomes a few statements of straight-line CUDA C++
// with all parameters as immediates, so a Gaussian leaf costs 2 FFMA per
// sample and no loads (features live in registers).  The source is compiled
// at prepare time to an sm_100a cubin (jit.cpp) -- no per-call host work.
//
// The generator builds a small SSA IR and prints it twice: as PTX (the
// product) and as plain C++ (used by the CPU test-suite to check the
// generator against the oracle without a GPU).
#pragma once
#include <stdint.h>

#include <string>
#include <vector>

#include "prepare.h"

namespace spnb {

struct JitOptions {
    int block = 256;             // threads per CTA (launch bound)
    int min_blocks = 2;          // __launch_bounds__ min CTAs per SM (register cap)
    int samples_per_thread = 1;  // K in 1..4: K interleaved copies of the body per thread
    int bar_every = 500;         // > 0: CTA barrier every bar_every IR instructions
                                 // (instruction-cache locality; C2 joint measured
                                 // 3.27e9 samples/s at 500 vs 2.88e9 without)
    int64_t task_cap_nodes = 3000;  // pack connected components up to this size
    int64_t max_task_nodes = 16000; // larger components: compiled path unsupported
                                    // (ptxas time and register spills grow with size)
    int64_t max_live_auto = 64;     // auto selection: larger ir_max_live stays on the
                                    // interpreter (RAT-SPN cross products: hundreds of live
                                    // values, ptxas takes minutes and the kernel spills)
    int space = 0;                  // value space (the deferred `probability`
                                    // type): 0 auto, 1 log2, 2 linear fp32 (discrete
                                    // leaves only, value range inside fp32's normal range)
};

struct JitTask {
    std::string name;            // kernel base name (spnb_t<i>); _j / _m suffixes
    std::string ptx[2];          // PTX modules for sm_100a: [0] entry <name>_j (joint),
                                 // [1] entry <name>_m (marginal); assembled in parallel
    std::string source;          // ptx[0] + ptx[1] (introspection)
    std::string cpp;             // the same IR as plain C++ (CPU tests): <name>_host(...)
    std::vector<int32_t> roots;  // output columns written by this task
    int64_t n_nodes = 0;         // canonical nodes evaluated (leaves included)
    int64_t n_features = 0;      // distinct features read
    int64_t max_live = 0;        // ir_max_live: inner values live at once (register pressure proxy)
};

struct JitProgram {
    std::vector<JitTask> tasks;
    std::vector<float> tables;   // discrete leaf tables (log2), read via `tab`
    bool fused_argmax = false;   // one task covers every root: argmax in-kernel
    bool linear = false;         // values are probabilities (linear fp32), tables hold p
    double lin_min = 0, lin_max = 0;  // linear: bounds of the non-zero values reachable
    // statistics (same definitions as PlanProgram)
    int64_t n_nodes = 0, n_leaves = 0, n_sums = 0, n_products = 0, n_sum_edges = 0;
    int64_t mufu_per_sample = 0, fma_per_sample = 0;
    int64_t mufu_exec_per_sample = 0;  // ex2 + lg2 the generated code executes
};

// Generate the compiled-path program.  Returns SPN_OK, or SPN_E_UNSUPPORTED
// (msg says why) when a connected component exceeds max_task_nodes.
int generate_jit(const GraphData &g, const JitOptions &opt, JitProgram &out, std::string &msg);

}  // namespace spnb
