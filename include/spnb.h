/*
 * spnb.h -- C ABI of the B200-native batched SPN inference library
 * (libspnb.so, built from paper_conf_cgo_sommera022_b200/csrc).
 *
 * The calls follow the paper's statement of the problem:
 *   - an SPN DAG of weighted sums, products and univariate leaves
 *     (Gaussian, categorical, histogram) plus its weights / leaf parameters
 *     comes in  (§II-A; HiSPN Table I);
 *   - a samples x features batch comes in (LoSPN batch_read, L80, L212-227;
 *     `numFeatures`, `inputType` of joint_query, L104-111);
 *   - one log-likelihood per sample per root goes out (L37; batch_write L304);
 *   - joint and marginal queries (`supportMarginal`, L108; marginal inference
 *     with partial evidence, L37, L394, L436-446);
 *   - the graph is kept separate from the query so one prepared plan serves
 *     both queries (L70: "keeping the representation of the DAG independent
 *     from the query ... allows to reuse the same graph").
 *
 * Conventions for every entry point:
 *   - all functions return int32 status: SPN_OK (0) or a negative SPN_E_*;
 *     spn_last_error() returns a thread-local message for the last failure;
 *   - no function keeps a pointer to caller memory after it returns;
 *   - "device pointer" means CUDA global memory on the plan's device;
 *   - output values are NATURAL logarithms (SPFlow convention, reading c4).
 */
#ifndef SPNB_H
#define SPNB_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* Node kinds (HiSPN Table I). */
enum spn_kind {
    SPN_GAUSSIAN    = 0, /* params {mean, stddev}, stddev > 0                  */
    SPN_CATEGORICAL = 1, /* params {p_0..p_{K-1}}, p_k in [0,1]; value index
                            = floor(x), valid iff 0 <= x < K (reading c3)      */
    SPN_HISTOGRAM   = 2, /* params {lb_0,ub_0,p_0, lb_1,ub_1,p_1, ...}: integer
                            half-open buckets [lb,ub), sorted, disjoint; p is
                            the probability of each integer in the bucket
                            (reading c2)                                        */
    SPN_SUM         = 3, /* weighted sum; weights[child_begin..] linear, >= 0,
                            used verbatim (reading c9)                          */
    SPN_PRODUCT     = 4  /* product of children                                 */
};

enum spn_status {
    SPN_OK            =  0,
    SPN_E_ARG         = -1, /* null pointer, negative size, bad handle type    */
    SPN_E_GRAPH       = -2, /* malformed graph (cycle, bad index, bad param)   */
    SPN_E_CUDA        = -3, /* CUDA runtime error (message has the CUDA text)  */
    SPN_E_OOM         = -4, /* host or device allocation failed                */
    SPN_E_UNSUPPORTED = -5  /* valid graph/option the library cannot run      */
};

/* One DAG node.  32 bytes, no padding.  Inner nodes use feature = -1. */
typedef struct spn_node {
    int32_t kind;        /* enum spn_kind                                      */
    int32_t feature;     /* leaf: input column in [0, n_features)              */
    int64_t child_begin; /* inner: first index into children[] / weights[]     */
    int64_t param_begin; /* leaf: first index into params[]                    */
    int32_t n_children;  /* inner: >= 1; leaf: 0                               */
    int32_t n_params;    /* leaf: see enum spn_kind; inner: 0                  */
} spn_node;

typedef struct spn_handle spn_handle; /* opaque: a graph or a prepared plan */

/* Options of spn_prepare (the analog of the paper's Python-exposed compiler
   knobs: block size, max partition size, ... PAPER.md L404, L481, L494). */
typedef struct spn_prepare_options {
    int32_t device;             /* CUDA device ordinal; -1 = current device    */
    int32_t block_threads;      /* threads per CTA, multiple of 32; 0 = auto
                                   (compiled path: 768, one CTA per SM;
                                   interpreter: from the feature tile size;
                                   layered path: 512 or 256, fixed)         */
    int32_t samples_per_thread; /* K in {1,2,4}; 0 = auto                      */
    int32_t layered_path;       /* 0 auto, 1 off (generic only), 2 force the
                                   tensor-core RAT-SPN path (E_UNSUPPORTED if
                                   the DAG is not a layered region graph)    */
    int64_t max_task_nodes;     /* partition cap in LoSPN ops;
                                   0 = auto (shared-memory budget), -1 = none  */
    int32_t tc_precision;       /* layered path: 0 auto, 1 f16 single pass, 2
                                   f16 hi/lo split (3 MMAs, ~fp32; v1 kernel).
                                   Auto: the v2 kernel's single pass with
                                   per-sample certification (spn_plan_stats
                                   cert_err); samples failing it are
                                   recomputed in hi/lo within the same call  */
    int32_t ctas_per_sm;        /* 0 = auto; compiled path: the kernels'
                                   __launch_bounds__ minimum CTAs per SM     */
    int32_t compiled_path;      /* 0 auto, 1 off (interpreter), 2 force: one
                                   straight-line kernel generated per SPN task
                                   (PTX) and assembled for the device at
                                   prepare time (the paper's per-SPN GPU
                                   compilation, §IV-C).
                                   Auto uses it for non-layered graphs unless
                                   samples_per_thread / max_task_nodes are set
                                   (interpreter knobs), a task keeps more than
                                   64 values live at once (register pressure:
                                   region-graph cross products) or
                                   compilation fails                          */
    int32_t layered_kernel;     /* layered path kernel: 0 auto (v2 when the
                                   region graph fits it, else v1), 1 v1
                                   (rat_eval.cu: one tile walks its schedule
                                   step by step), 2 v2 (rat2.cu: warp-
                                   specialised leaf / MMA / epilogue roles;
                                   E_UNSUPPORTED if not applicable)          */
    int32_t value_space;        /* compiled path: 0 auto, 1 log2 space, 2 linear
                                   fp32 (the paper's deferred `probability`
                                   datatype choice).  Auto picks
                                   linear when every leaf is discrete and
                                   interval bounds keep every non-zero value
                                   in [2^-100, 2^100]: sums become FFMA chains
                                   and the only MUFU op is one lg2 per root.
                                   2 on an ineligible graph: E_UNSUPPORTED  */
    int32_t leaf_tc;            /* layered v2: leaf layer on the tensor cores
                                   (one GEMM of per-sample features x~^2, x~
                                   against the Gaussians' expanded constants,
                                   f16 hi/lo split, fp32 accumulation in TMEM).
                                   0 auto (= off: measured slower than the FMA
                                   leaves on C4/C5), 1 off
                                   (FP32 FMA leaves), 2 on (needs tc_precision
                                   0: the certification recomputes inputs
                                   outside the split's range; E_UNSUPPORTED if
                                   not applicable)                           */
    int32_t reserved[4];        /* must be zero                                */
} spn_prepare_options;

/* Statistics of a prepared plan (used by the benchmark's roofline). */
typedef struct spn_plan_stats {
    int64_t n_nodes;            /* after canonicalisation                     */
    int64_t n_leaves, n_sums, n_products;
    int64_t n_sum_edges;
    int64_t n_tasks;            /* partitions (§IV-A4); 1 on the
                                   layered path (it does not partition)       */
    int64_t n_cut_values;       /* values crossing tasks (stored+loaded once) */
    int64_t partition_cost;     /* sum over values of #consuming other tasks  */
    int64_t n_records;          /* interpreter records over all tasks;
                                   layered path: schedule steps per tile      */
    int64_t n_global_slots;     /* per-warp scratch slots (global memory)     */
    int64_t n_smem_slots;       /* per-warp scratch slots (shared memory)     */
    int64_t max_stack;          /* deepest register-stack position used       */
    int64_t mufu_per_sample;    /* algorithmic: sum over sums of the fan-in
                                   (max-shifted n-ary LSE: the shift term is
                                   exactly 1, so n-1 ex2 + 1 lg2; 0 for a
                                   single child); layered path: na + nb + S
                                   per sum region (the exps and lg2s)         */
    int64_t fma_per_sample;     /* algorithmic FP32 ops (2/leaf, 1/prod edge,
                                   3/sum edge)                                */
    int64_t bytes_per_sample;   /* 4*n_features + 4*n_roots (+4 argmax)       */
    int64_t tc_flops_per_sample;/* layered path only                          */
    int32_t path;               /* 0 generic interpreter, 1 layered RAT path,
                                   2 compiled (generated per-SPN kernels)    */
    int32_t block_threads, samples_per_thread, grid;
    int32_t smem_bytes;
    int32_t x_in_smem;
    double  prepare_ms;
    /* compiled path (path 2) */
    int32_t kernel_regs;        /* max registers per thread over the kernels  */
    int32_t ctas_per_sm;        /* min resident CTAs per SM over the kernels  */
    int64_t mufu_exec_per_sample; /* ex2 + lg2 the generated code executes    */
    double  compile_ms;         /* PTX assembly wall time (tasks in parallel)  */
    int64_t chunk_samples;      /* layered path: samples per transposed chunk
                                   (one transpose + one layered launch each)  */
    int32_t layered_kernel;     /* layered path: 1 v1, 2 v2 (0 other paths)   */
    int32_t tc_passes;          /* layered path: f16 MMA passes (1 or 3)      */
    int32_t value_space;        /* 1 log2 space, 2 linear fp32 (compiled path) */
    int32_t certified;          /* layered v2, tc_precision auto: 1 when every
                                   sample's single-pass result is checked
                                   against cert_err and failures recomputed in
                                   hi/lo precision (v1 kernel)                */
    double  cert_err;           /* layered v2: a-priori bound (nats) on the
                                   single f16 pass's deviation from the exact
                                   contraction, for every root; a sample is
                                   kept when cert_err <= 0.9e-4 max(1, |ln p|
                                   - cert_err) for all its roots (the other
                                   0.1e-4 of the tolerance covers the fp32
                                   arithmetic both precisions share)          */
    int32_t leaf_tc;            /* layered v2: 1 when the leaf layer runs on
                                   the tensor cores (spn_prepare_options)    */
} spn_plan_stats;

/* Fill *opt with defaults (all auto). */
void spn_default_options(spn_prepare_options *opt);

/*
 * Validate and COPY a graph (the caller may free its arrays on return).
 *   nodes[n_nodes]; children[n_edges] are node indices; weights[n_edges]
 *   are linear sum weights (ignored for product edges); params[n_params];
 *   roots[n_roots] node indices (one output column per root, in order).
 * Errors: SPN_E_ARG (null pointer with non-zero size, negative sizes,
 *   n_roots < 1, n_features < 1), SPN_E_GRAPH (child/root/feature index out
 *   of range, inner node without children, leaf with children, cycle,
 *   stddev <= 0 or non-finite, probability outside [0,1] or NaN, negative or
 *   NaN weight, malformed/non-integer/overlapping histogram buckets,
 *   wrong n_params).  On error *out_graph is left NULL.
 */
int spn_load_graph(const spn_node *nodes, int64_t n_nodes,
                   const int64_t *children, const double *weights, int64_t n_edges,
                   const double *params, int64_t n_params,
                   const int64_t *roots, int32_t n_roots, int32_t n_features,
                   spn_handle **out_graph);

/*
 * Prepare a graph for inference on opt->device (host work once per graph,
 * the analog of the paper's compilation, §IV-A): canonicalise (drop
 * single-input nodes, L330), level and order the DAG, partition it into
 * tasks (acyclic partitioning with 1% slack and per-value cut cost, L336-346),
 * emit the per-task node programs, pack parameters (log2 domain) and upload
 * them (device memory owned by the plan).  The plan keeps no reference to
 * the graph; either may be freed first.  opt may be NULL (defaults).
 * Errors: SPN_E_ARG, SPN_E_CUDA, SPN_E_OOM, SPN_E_UNSUPPORTED.
 */
int spn_prepare(const spn_handle *graph, const spn_prepare_options *opt,
                spn_handle **out_plan);

/*
 * Joint log-likelihood (full evidence), asynchronous on cuda_stream
 * (cudaStream_t; NULL = legacy default stream).
 *   x       device, [n][ld] fp32 row-major, ld >= n_features (read only)
 *   out     device, [n][n_roots] fp32 row-major: ln p_r(x_s)
 *   argmax  device, [n] int32, nullable: lowest root index with the largest
 *           non-NaN out[s][r], -1 if all NaN
 * n = 0 is a no-op.  NaN in x yields NaN for every root depending on that
 * feature (reading c7).  Argument and launch errors are returned
 * synchronously; faults inside the kernel surface at the caller's next sync.
 * Re-entrant for distinct streams: the plan's tables are read-only, and its
 * scratch (transposed features of the layered path, global slots of the
 * interpreter) is used by one launch at a time -- a call on a different
 * stream than the previous call makes its stream wait for the previous
 * call's completion event first (calls on one stream are stream-ordered).
 */
int spn_infer_joint(spn_handle *plan, const float *x, int64_t n, int64_t ld,
                    float *out, int32_t *argmax, void *cuda_stream);

/*
 * Marginal log-likelihood: identical to spn_infer_joint except that NaN
 * entries of x are missing evidence and the leaf reading them contributes
 * log 1 = 0 (PAPER.md L37 partial evidence; reading c6).  Without NaNs the
 * result is bitwise identical to spn_infer_joint.
 */
int spn_infer_marginal(spn_handle *plan, const float *x, int64_t n, int64_t ld,
                       float *out, int32_t *argmax, void *cuda_stream);

/*
 * End-to-end variants with HOST buffers (x_host [n][ld], out_host
 * [n][n_roots], argmax_host nullable [n]): the library stages chunks through
 * device buffers it owns, overlapping host->device copies, inference and
 * device->host copies on its own streams (the paper's host<->device data
 * movement, >60% of GPU time, L448-454).  Synchronous: returns when out_host
 * is filled.  Pinned (page-locked) host memory gives full overlap.
 * Certified layered plans (spn_plan_stats.certified) keep whole groups of up
 * to ~4 GB of rows on the device (allocated on first use, freed with the
 * plan): rows land in pieces of one tile per SM, each piece's kernel starts
 * when its rows are in, and the group ends with one certification round and
 * one copy of its outputs, so the result equals spn_infer_* on the same rows
 * bit for bit.
 */
int spn_infer_joint_host(spn_handle *plan, const float *x_host, int64_t n, int64_t ld,
                         float *out_host, int32_t *argmax_host);
int spn_infer_marginal_host(spn_handle *plan, const float *x_host, int64_t n, int64_t ld,
                            float *out_host, int32_t *argmax_host);

/* Plan statistics.  SPN_E_ARG if h is not a plan. */
int spn_plan_info(const spn_handle *plan, spn_plan_stats *stats);

/*
 * Host-only introspection (no GPU needed; used by the CPU test-suite).
 *
 * spn_partition_graph: run canonicalisation + the acyclic partitioner
 *    with cap max_task_ops (LoSPN operations; <= 0 means
 *   one task) and report, per ORIGINAL node, its task id (-1 for leaves and
 *   for nodes removed by canonicalisation).  task_of_node[n_nodes] caller
 *   owned.  *n_tasks, *cost (sum over values of the number of other tasks
 *   consuming them, reading c12) and *cut_values may be NULL.
 *
 * spn_build_program: run the whole preparer for samples_per_thread K and
 *   feature staging x_in_smem (tile stride 32K+4) without touching a GPU and
 *   copy out the node program.  Call with NULL buffers to get the sizes:
 *   *n_records (16-byte records, program.h format), *n_tasks (task_off has
 *   n_tasks+1 entries), *n_tables (floats), *n_edges (16-byte GLSE terms),
 *   then again with buffers of at least those sizes.  slots[0] receives the
 *   number of shared-memory slots, slots[1] global slots, slots[2] the max
 *   stack depth.
 */
/*
 * spn_build_layered: run the layered (RAT-SPN region graph) detector and
 *   plan builder of the tensor-core path without a GPU.  Returns SPN_OK and
 *   *is_layered = 0/1 (why[why_len] receives the reason when 0).  With NULL
 *   buffers only the sizes are returned: sizes[0] steps (each
 *   sizeof_step bytes), sizes[1] vars (int32), sizes[2] fparams (float),
 *   sizes[3] weight-image bytes, sizes[4] roots, sizes[5] activation floats,
 *   sizes[6] sizeof_step.  Then call again with buffers of those sizes.
 */
int spn_build_layered(const spn_handle *graph, int32_t *is_layered, char *why, int64_t why_len,
                      int64_t *sizes, void *steps, int32_t *vars, float *fparams, void *wimg,
                      int32_t *root_map);
/*
 * spn_build_layered2: the same for the v2 kernel's plan (rat2.cu; requires a
 *   complete binary region tree per repetition, uniform leaf width I (a
 *   multiple of 8, <= 48) and sum width S <= 48).  *ok = 0/1 (why[] gets the
 *   reason).  sizes[0] steps (sizes[5] bytes each), sizes[1] vars (int32),
 *   sizes[2] fparams (float), sizes[3] weight-image bytes, sizes[4] roots;
 *   dims[11] = {F, C, I, S, D, gcols, kpad_bot, kpad_up, max_wgroup,
 *   max_vars, max_blk}.  NULL buffers: sizes and dims only.
 *   *tc_err_1pass (nullable) receives the plan's a-priori bound (nats) on
 *   the single f16 pass's deviation from the exact contraction.
 */
int spn_build_layered2(const spn_handle *graph, int32_t *ok, char *why, int64_t why_len,
                       int64_t *sizes, int32_t *dims, void *steps, int32_t *vars, float *fparams,
                       void *wimg, int32_t *root_map, double *tc_err_1pass);
/*
 * spn_build_layered2_ex: spn_build_layered2 with leaf_tc = 1 building the
 *   tensor-core leaf variant (spn_prepare_options.leaf_tc): per leaf step
 *   fparams holds the centres M[lvp] and the weight-image bytes at w_off
 *   hold the joint parameter image [hi, lo] (wbytes_a bytes each, K = kl_j)
 *   then the marginal one (wbytes_b each, K = kl_m), both K-major f16 with
 *   48 rows; dims[14] = dims[11] of spn_build_layered2 then {lvp, kl_j,
 *   kl_m}.  leaf_tc = 0: exactly spn_build_layered2 (dims[11]).
 */
int spn_build_layered2_ex(const spn_handle *graph, int32_t leaf_tc, int32_t *ok, char *why,
                          int64_t why_len, int64_t *sizes, int32_t *dims, void *steps, int32_t *vars,
                          float *fparams, void *wimg, int32_t *root_map, double *tc_err_1pass);
int spn_partition_graph(const spn_handle *graph, int64_t max_task_ops, int32_t *task_of_node,
                        int32_t *n_tasks, int64_t *cost, int64_t *cut_values);
int spn_build_program(const spn_handle *graph, int32_t samples_per_thread, int32_t x_in_smem,
                      int64_t max_task_ops, int64_t smem_slot_cap,
                      void *records, int64_t *n_records, int64_t *task_off, int64_t *n_tasks,
                      float *tables, int64_t *n_tables, void *edges, int64_t *n_edges,
                      int64_t *slots);

/*
 * spn_codegen: run the compiled path's code generator (no GPU needed) and
 *   return task `task`'s generated code: lang = 1 the PTX the library
 *   assembles (entries <name>_j / <name>_m), lang = 0 the same IR printed as
 *   plain C++ defining `<name>_host(x, n, ld, out, R, argmax, tab, marg)`,
 *   which the CPU test-suite compiles to check the generator against the
 *   oracle.  Bits 8..9 of lang select the value space (0 auto, 1 log2,
 *   2 linear; see spn_prepare_options.value_space).
 *   Sizes first (NULL buffers): *src_len (bytes incl. NUL),
 *   *n_roots, *n_tables (floats), *n_tasks; then again with buffers.
 *   name[64] receives the kernel base name; roots[] the output columns the
 *   task writes; tables[] the discrete-leaf tables (log2) passed as `tab`.
 *   compile = 1 additionally assembles the PTX with nvJitLink for
 *   sm_<arch> (arch e.g. "100a"), returning SPN_E_UNSUPPORTED with the
 *   assembler log in spn_last_error on failure.
 */
int spn_codegen(const spn_handle *graph, int32_t task, int32_t lang, char *src, int64_t *src_len,
                char *name, int32_t *roots, int32_t *n_roots, float *tables, int64_t *n_tables,
                int32_t *n_tasks, int32_t compile, const char *arch);

/* Free a graph or a plan; NULL is a no-op.  The caller must synchronise
   outstanding work on the plan first. */
void spn_free(spn_handle *h);

/* Thread-local message for the last non-OK status ("" if none). */
const char *spn_last_error(void);

#ifdef __cplusplus
}
#endif
#endif /* SPNB_H */
