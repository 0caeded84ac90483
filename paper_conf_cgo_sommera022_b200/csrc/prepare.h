// prepare.h -- host-side graph preparer (the analog of SPNC's
// target-independent compilation steps, §IV-A).
#pragma once
#include <stdint.h>

#include <string>
#include <vector>

#include "program.h"

namespace spnb {

// Validated private copy of a graph (spn_load_graph).
struct GraphData {
    int32_t F = 0;
    std::vector<int32_t> kind, feature, n_children, n_params;
    std::vector<int64_t> child_begin, param_begin, children, roots;
    std::vector<double> weights, params;
};

struct CodegenConfig {
    int K = 4;                 // samples per thread
    bool x_in_smem = true;     // features staged in shared memory
    int tpw = 132;             // per-warp tile stride (floats) when x_in_smem
    int64_t max_task_ops = -1; // partition cap (LoSPN ops); <= 0: single task
    int64_t smem_slot_cap = 0; // shared-memory slots available per warp
    int lse_max = 4;           // largest stack LSE fan-in
    int maxd = MAXD;           // register-stack depth of the kernel variant
};

struct PlanProgram {
    std::vector<Rec> prog;
    std::vector<int64_t> task_off;  // n_tasks + 1
    std::vector<float> tables;
    std::vector<Edge> edges;
    int64_t n_gslots = 0;
    int64_t n_sslots = 0;
    int64_t max_stack = 0;
    int64_t max_task_records = 0;
    // statistics
    int64_t n_nodes = 0, n_leaves = 0, n_sums = 0, n_products = 0, n_sum_edges = 0;
    int64_t n_cut_values = 0, partition_cost = 0;
    int64_t mufu_per_sample = 0, fma_per_sample = 0;
    int64_t n_roots = 0;
};

// Canonical DAG: reachable nodes in post-order (children first), single-input
// nodes removed where exact (products always; sums only if the weight is 1).
struct CGraph {
    int64_t n = 0;
    std::vector<int32_t> kind;
    std::vector<int64_t> orig;          // original node id
    std::vector<int64_t> cb;            // CSR children
    std::vector<int64_t> ch;
    std::vector<double> w;
    std::vector<int64_t> pb;            // CSR parents
    std::vector<int64_t> par;
    std::vector<std::vector<int32_t>> rootrefs;
};
void canonicalise(const GraphData &g, CGraph &c);

// Returns 0 or a negative spn_status with msg set.
int validate_graph(const GraphData &g, std::string &msg);

// Canonicalise, level, partition, generate per-task programs, pack tables.
int build_program(const GraphData &g, const CodegenConfig &cfg, PlanProgram &out,
                  std::string &msg);

// ---- partitioner (exposed for tests through the C ABI debug hook) --------
struct PartitionResult {
    std::vector<int32_t> task;   // per inner node (canonical ids), -1 for leaves
    int32_t n_tasks = 1;
    int64_t cost = 0;            // sum over values of #consuming other tasks
    int64_t cut_values = 0;
};

int partition_graph(const GraphData &g, int64_t cap, std::vector<int32_t> &task_of_orig,
                    PartitionResult &res);

}  // namespace spnb
