// layered.h -- detection of layered (RAT-SPN-style) region-graph structure
// in a flat SPN DAG and the plan of the tensor-core path (kernel KB/KC).
//
// A layered SPN (§V-B: RAT-SPNs, "random tensorized"
// region graphs) consists of
//   * leaf regions: I "distributions", each a product of Gaussian leaves over
//     the region's variable set (or a single Gaussian leaf);
//   * partitions: the cross product of two child regions' values (product
//     nodes with exactly two children, one per child region);
//   * sum regions: S weighted sums over all products of one partition;
//   * the root region: the graph roots, C sums over the products of one or
//     more partitions (one per repetition).
// Every region feeds exactly one partition (a tree of regions per
// repetition).  The preparer recognises this structure from the DAG alone.
#pragma once
#include <stdint.h>

#include <string>
#include <vector>

#include "prepare.h"

namespace spnb {

// One step of the per-tile schedule (see rat_eval.cu).
struct LStep {
    int32_t type;        // 0 LEAF, 1 SUM, 2 ROOT
    int32_t n_out;       // values produced (I, S or C)
    int32_t na, nb;      // child region sizes (SUM / ROOT)
    int32_t buf_a, buf_b, buf_out;  // shared-memory buffer offsets (floats)
    int32_t k_pad;       // nb rounded up to 16 (f16 K-step)
    int32_t s_per_group; // sums per N-group
    int32_t n_groups;
    int32_t n_group;     // N columns per group (multiple of 16)
    int32_t n_vars;      // LEAF: variables of the region
    int64_t vars_off;    // LEAF: int32 offset into vars[]
    int64_t par_off;     // LEAF: float offset of the staged block: (a, b)[n_vars][n_out], C[n_out]
    int64_t cst_off;     // LEAF: float offset of C[n_out] (inside the block)
    int64_t w_off;       // SUM/ROOT: byte offset of the f16 weight images; LEAF: block floats
    int64_t w_group_bytes;  // bytes per (group, part) image
    int32_t rep;         // LEAF: index of the next LEAF step in the schedule (-1: none)
    int32_t pad_;
};

struct LayeredPlan {
    bool ok = false;
    std::string why;             // reason when not layered
    int32_t F = 0, C = 0, R = 0; // features, classes (roots), repetitions
    std::vector<LStep> steps;
    std::vector<int32_t> vars;
    std::vector<float> fparams;  // leaf (a,b) pairs and C constants
    std::vector<uint16_t> wimg;  // f16 weight images (hi then lo per group)
    int32_t smem_floats = 0;     // activation buffers
    int32_t max_kpad = 0, max_ngroup = 0, max_na = 0, max_vars = 0;
    int32_t max_leaf_params = 0;    // floats of the largest staged leaf parameter block
    int32_t first_leaf = -1;
    std::vector<int32_t> root_map;  // root-region value index -> output column
    int64_t tc_flops_per_sample = 0;  // one precision pass
    int64_t fma_per_sample = 0;
    int64_t mufu_per_sample = 0;
    int64_t n_leaf_regions = 0, n_sum_regions = 0;
    // region tree kept for the v2 kernel (rat2.cu): per step the child steps
    // (SUM / ROOT) and the unpacked parameters -- SUM / ROOT: linear weights
    // W[s][i][j] (na x nb cells per sum); LEAF: a[v][i], b[v][i] (log2-domain
    // Gaussian constants, log2 N = c - (a x - b)^2) then C[i] = sum_v c_vi
    std::vector<int32_t> child_a, child_b;
    std::vector<std::vector<double>> raw;
    // weight range (the v1 kernel stores weights unscaled as f16 hi/lo: a
    // weight >= 65504 would be inf, a non-zero one < 2^-24 would flush to 0)
    double w_min_nz = 0.0, w_max = 0.0;
};

// ---------------------------------------------------------------- v2 plan
// Plan of the warp-specialised layered kernel (rat2.cu).  Accepted when
// every repetition is a complete binary region tree whose partitions pair
// either two leaf regions ("BOT") or two sum regions ("UP"), with uniform
// leaf-region width I (multiple of 4, <= 48) and sum-region width S.
struct R2Step {
    int32_t type;        // 0 LEAF, 1 BOT (children: two leaf regions), 2 UP (two sum regions)
    int32_t root;        // 1: the outputs are root (class) values, accumulated over repetitions
    int32_t n_out, na, nb, kpad;
    // N groups alternate between the two TMEM accumulators: even groups
    // (buffer A, R2_COLS_A columns) hold spg_a sums, odd groups (buffer B)
    // spg_b; the last pair may be partial (a group may be empty); n_groups
    // is even.  ncol_*: MMA N (sums x na rounded up to 16)
    int32_t n_groups, spg_a, ncol_a, spg_b, ncol_b;
    int32_t slot_a, slot_b, slot_out;        // TMEM activation slots (1-based; UP inputs, output)
    int32_t n_vars;      // LEAF: variables of the region
    int32_t pad_;
    int64_t vars_off;    // LEAF: int32 offset into vars
    int64_t blk_off;     // LEAF: float offset of the block (a,b)[v][I], C[I] (tensor-core
                         // leaves: the per-variable centres M[lvp]); SUM: kscale[n_out]
    int64_t blk_floats;  // LEAF: block size in floats (multiple of 4)
    int64_t w_off;       // SUM: byte offset of the images: per group pair [A hi, A lo, B hi, B lo]
                         // LEAF (tensor-core leaves): joint image [hi, lo], then marginal [hi, lo]
    int64_t wbytes_a, wbytes_b;  // bytes of one part image of an A / B group (LEAF: joint / marginal)
};
constexpr int R2_COLS_A = 240, R2_COLS_B = 160;  // TMEM accumulator buffers (columns)
// tensor-core leaf layer: narrower sum accumulators make room for the leaf
// accumulator (N = 48 >= I) in TMEM
constexpr int R2T_COLS_A = 160, R2T_COLS_B = 160, R2T_COLS_L = 48;

struct Rat2Plan {
    bool ok = false;
    std::string why;
    int32_t F = 0, C = 0, I = 0, S = 0, D = 0;  // D: TMEM activation slots used (1..D)
    int32_t max_vars = 0, max_blk = 0;          // largest leaf region / parameter block (floats)
    int32_t kpad_bot = 0, kpad_up = 0;          // K of the BOT / UP contractions (x16)
    int32_t max_wgroup = 0;                     // bytes of the largest (group, part) image
    int32_t gcols = 0;                          // TMEM columns before the activation slots
    int32_t cols_a = 0, cols_b = 0;             // accumulator widths (R2_COLS_* / R2T_COLS_*)
    int32_t ea_max = 0;                         // max(I, S) rounded up to 8
    // tensor-core leaf layer (leaf_tc): a leaf region's log-densities are one
    // GEMM L[m, i] = sum_k F[m, k] P[k, i] over the per-sample features
    // F = (x~^2, x~) per variable (x~ = x - M_v, hi/lo f16 split) plus a
    // constant column (joint) or per-variable observed indicators
    // (marginal); P holds -a^2, 2 a b~ and c - b~^2 (PAPER.md L128-167
    // Gaussian, expanded around the centre M_v: b~ = b - a M_v)
    bool leaf_tc = false;
    int32_t lvp = 0;                            // variables per region rounded up to 4
    int32_t kl_j = 0, kl_m = 0;                 // K of the joint / marginal leaf GEMM (x16)
    std::vector<R2Step> steps;
    std::vector<int32_t> vars;
    std::vector<float> fparams;                 // leaf blocks, then per-sum scale exponents
    std::vector<uint16_t> wimg;                 // f16 images
    std::vector<int32_t> root_map;
    int64_t n_leaf = 0, n_sum = 0;
    // a-priori bound (natural log units) on |ln p(1 f16 pass) - ln p(exact
    // contraction)| for every root: per sum, the exact relative rounding of
    // its f16 weights, the f16 rounding of the B-side exps (2^-11, normal
    // range by the 2^15 shift), the flushed exps below 2^-29 (2^-29 times
    // sum/min weight) and fp32 accumulation; propagated bottom-up (a
    // product adds its children's bounds, a sum adds its own, LSE being
    // 1-Lipschitz in the max norm).  Infinite if a sum has a zero weight.
    double tc_err_1pass = 0.0;
};

// Builds the v2 plan from a detected layered plan; fails (ok = false, why)
// when the structure is outside the v2 kernel's constraints.
// leaf_tc: tensor-core leaf layer (fails when a leaf constant or centre is
// outside the f16 range of the split operands).
void build_rat2(const LayeredPlan &lp, Rat2Plan &p, bool leaf_tc = false);

// Kernel parameters of rat2_kernel.
struct R2Params {
    const R2Step *steps;
    int32_t n_steps;
    int32_t C, I, S;
    const int32_t *vars;
    const float *fparams;
    const uint8_t *wimg;
    const int32_t *root_map;
    const float *xT;      // transposed features [F][ldT]
    int64_t ldT;
    int64_t n;            // samples in this launch (rows of xT used)
    float *out;
    int32_t *argmax;
    int32_t prec;         // 1: one f16 pass; 3: hi/lo split (3 MMAs)
    int32_t max_vars, max_blk, kpad_bot, kpad_up, max_wgroup, gcols, D;
    // tensor-core leaf layer: K of the leaf GEMM (joint / marginal), vars
    // rounded up to 4, feature image (hi part, lo part follows) and the
    // offset of the parameter image inside an input slot
    int32_t lvp, kl_j, kl_m, off_f, f_bytes, pimg_off;
    int32_t n_in, n_w;    // ring depths: leaf inputs, weight groups
    // shared-memory carve-up (byte offsets, computed on the host)
    int32_t off_in, in_bytes, off_ea, ea_bytes, off_bimg, bimg_bytes, off_uimg, uimg_bytes,
        off_w, w_bytes, off_bar;
    int32_t smem_bytes;
    unsigned long long *prof;  // optional: per-role phase cycles [4 roles][8] (SPNB_PROFILE)
    // certification of the single f16 pass (tc_precision auto): a sample
    // whose roots do not all satisfy cert_err <= cert_tol * max(1, |ln p| -
    // cert_err) is appended to flag_idx (global row = row0 + tile row) for
    // the hi/lo recomputation; flag_count == nullptr: no certification
    float cert_err, cert_tol;
    int32_t *flag_count;
    int64_t *flag_idx;
    int64_t row0;
};

// Detects the structure; on success fills plan (ok = true).
// n_cap: largest N (columns) of one MMA group (<= 240).
void detect_layered(const GraphData &g, LayeredPlan &plan, int n_cap = 240);

// Kernel parameters of rat_eval_kernel (rat_eval.cu), filled by api.cpp.
struct RParams {
    const LStep *steps;
    int32_t n_steps;
    int32_t C;
    const int32_t *vars;
    const float *fparams;
    const uint8_t *wimg;
    const int32_t *root_map;
    const float *xT;
    int64_t ldT;
    int64_t n;
    float *out;
    int32_t *argmax;
    int32_t prec;       // 1: single f16 pass; 3: hi/lo split
    int32_t smem_floats, max_kpad, max_ngroup, max_na;
    int32_t max_vars;   // largest leaf region (staged x rows)
    int32_t first_leaf; // index of the first LEAF step
    int32_t max_leaf_params;  // floats of the largest staged leaf parameter block
    int32_t wbufs;      // 2: double-buffered weight groups; 1: single buffer
    int32_t overlap;    // 1 (with wbufs 2): epilogue of group g-1 under MMA g (TMEM
                        // ping-pong, default); 0: MMA g, then its epilogue.  Measured
                        // on C4: 5.78e6 vs 5.45e6 samples/s with 16 warps (TMEM reads
                        // under a running MMA are slower, but the MMA is hidden)
    unsigned long long *prof;  // optional phase-cycle counters (thread 0 of each CTA)
    // optional device-side sample count (the certification fallback): when
    // set, n = clamp(*n_count - n_off, 0, n) is read by the kernel itself
    const int32_t *n_count;
    int64_t n_off;
};

}  // namespace spnb
