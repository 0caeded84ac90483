// program.h -- the node-program format shared by the host preparer and the
// sm_100a interpreter kernel (dag_eval.cu).  Internal to libspnb.
//
// A plan is a sequence of TASKS (the paper's LoSPN Tasks, PAPER.md L78-80,
// L336-346).  Each task is a list of 16-byte records executed once per sample
// by every thread for its K samples, over a register STACK of depth <= MAXD
// (values in the log2 domain).  Record word x = case | arg << 9 where
// case = op * 17 + sp and sp = stack depth BEFORE the op (0..16); y, z, w are
// operands.  The static sp lets the kernel keep the stack in registers: every
// (op, sp) pair is its own case of one dense switch (a single jump table), with
// constant register indices.  Feature and slot operands are byte offsets
// pre-multiplied by the preparer (feature * 4 * tile stride, slot * 128 * K).
// Sum weights are folded into the records producing the children ("bias"),
// so the LSE records carry no weights.
//
//   LPUSH  ng | C, nd        r[sp]   = C + sum of ng Gaussian + nd discrete leaves
//   LACC   ng | C, nd        r[sp-1] += (same)          (leaf children of a product)
//   GPUSHn / GACCn  | C, f0|f1<<16, f2|f3<<16   same for exactly n <= 4 Gaussian
//                            leaves (no loop); the 16-bit feature offsets of the
//                            leaves ride in the header so x loads issue at once
//   SLPk  counts | bias, C0, C1   r[sp] = LSE_c(C_c + sum of n_c Gaussian leaves) + bias
//       for k = 2..4 children (n_c in 1..7 packed 3 bits each in arg); for k >= 3
//       a record {C2, C3} follows, then the children's parameter records.
//   SLPU2 | bias, C0, C1  + {f0|f1<<16, f2|f3<<16, -, -} + 4 leaf records
//   SLPU3 | bias, C0, C1  + {C2, f0|f1<<16, f2|f3<<16, f4|f5<<16} + 6 leaf records
//       straight-line forms of the dominant SLP shapes (children of 2 leaves),
//       with the leaves' feature offsets up front so all loads issue at once.
//       followed by ng Gaussian parameter records {f, a, b, c} and nd discrete
//       records {f, table, lo, K}.  Gaussian: c - (a*x_f - b)^2 = log2 N(x; mu, s)
//       with a = 1/(s sqrt(2 ln2)), b = a mu, c = -log2(s sqrt(2 pi)); the c's
//       (and the bias) are pre-summed into C, so a leaf costs 2 FFMA: t = a x - b,
//       acc -= t*t.  Marginal kernels subtract c instead of t^2 for a NaN input
//       (log 1 = 0).  Discrete: x in [lo, lo+K) ? table[floor(x)-lo] : -inf.
//   ADD      | bias          r[sp-2] += r[sp-1] + bias           product edge
//   LSE1..4  | bias          r[sp-n] = LSE_i(r[sp-n+i]) + bias   weighted sum: the
//                            largest input is the shift m, so its ex2(0)=1 needs no
//                            MUFU: n-1 ex2 + 1 lg2 per sum
//   LDS/LDG s | bias         r[sp]   = slot_s + bias   (shared / global scratch;
//                            LDG/STG carry the slot's byte offset in z, 32 bits)
//   STS/STG s                slot_s  = r[sp-1]  (the next record's sp pops)
//   GLSE     | off_lo, off_hi, n   r[sp] = LSE over edge terms slot(a)[+slot(b)]+lw
//   OUT    r                 out[., r] = ln2 * r[sp-1]
//   END
#pragma once
#include <stdint.h>

namespace spnb {

enum Op : uint32_t {
    OP_END = 0,
    OP_LPUSH = 1,   // generic leaf product (loop; Gaussian + discrete leaves)
    OP_LACC = 2,
    OP_ADD = 3,
    OP_LSE1 = 4,
    OP_LSE2 = 5,
    OP_LSE3 = 6,
    OP_LSE4 = 7,
    OP_LDS = 8,
    OP_LDG = 9,
    OP_STS = 10,
    OP_STG = 11,
    OP_GLSE = 12,
    OP_OUT = 13,
    OP_NOP = 14,
    OP_GPUSH1 = 15, // straight-line products of 1..4 Gaussian leaves
    OP_GPUSH2 = 16,
    OP_GPUSH3 = 17,
    OP_GPUSH4 = 18,
    OP_GACC1 = 19,
    OP_GACC2 = 20,
    OP_GACC3 = 21,
    OP_GACC4 = 22,
    OP_SLP2 = 23,   // fused weighted sum of 2..4 Gaussian leaf products
    OP_SLP3 = 24,
    OP_SLP4 = 25,
    OP_SLPU2 = 26,  // straight-line SLP: 2 children x 2 Gaussian leaves
    OP_SLPU3 = 27,  // straight-line SLP: 3 children x 2 Gaussian leaves
    OP_COUNT = 28
};

constexpr int MAXD = 16;              // register stack depth
constexpr uint32_t ARG_BITS = 23;
constexpr uint32_t CASE_BITS = 9;
constexpr uint32_t NSP = MAXD + 1;     // sp values 0..MAXD
constexpr uint32_t ARG_MAX = (1u << ARG_BITS) - 1;
constexpr uint32_t SLOT_NONE = 0xFFFFFFFFu;
constexpr uint32_t SLOT_GLOBAL = 0x80000000u;  // flag in GLSE edge slot refs

struct alignas(16) Rec {
    uint32_t x, y, z, w;
};

inline Rec make_rec(uint32_t op, uint32_t sp, uint32_t arg, uint32_t y = 0,
                    uint32_t z = 0, uint32_t w = 0) {
    Rec r;
    r.x = (op * NSP + sp) | (arg << CASE_BITS);
    r.y = y;
    r.z = z;
    r.w = w;
    return r;
}

// GLSE edge term: value = slot(a) [+ slot(b)] + lw  (b == SLOT_NONE if absent)
struct alignas(16) Edge {
    uint32_t a, b;
    float lw;
    uint32_t pad;
};

// Kernel launch parameters (POD, passed by value).
struct KParams {
    const Rec *prog;            // all tasks, concatenated
    const int64_t *task_off;    // [n_tasks + 1] record offsets (device)
    int32_t n_tasks;
    int32_t prog_cap;           // shared-memory program buffer (records)
    int32_t first_task_len;     // records of task 0 (single-task fast path)
    const float *tables;        // discrete leaf tables, log2 values
    const Edge *edges;          // GLSE terms
    const float *x;
    int64_t n;
    int64_t ld;
    int32_t F;
    int32_t R;
    float *out;
    int32_t *argmax;
    float *gslots;              // [total_warps][n_gslots][32*K]
    int32_t n_gslots;
    int32_t n_sslots;           // shared-memory slots per warp
    int32_t x_in_smem;
    int32_t tpw;                // padded per-warp tile stride (floats)
    int64_t n_wtiles;           // ceil(n / (32*K))
};

}  // namespace spnb
