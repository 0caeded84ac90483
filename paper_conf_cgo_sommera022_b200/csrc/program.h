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
// constant register indices.  Feature and slot operands are pre-multiplied by
// the preparer into float offsets (feature * tile stride, slot * 32K).
//
//   GPUSH  f | a, b, c      r[sp]   = c - (a*x_f - b)^2         Gaussian leaf
//   GACC   f | a, b, c      r[sp-1] += c - (a*x_f - b)^2        leaf into product
//   DPUSH  f | tab, lo, K   r[sp]   = x in [lo,lo+K) ? tab[floor(x)-lo] : -inf
//   DACC   f | tab, lo, K   r[sp-1] += (same)                   discrete leaf
//   ADD                     r[sp-2] += r[sp-1]                   product edge
//   LSE1..4  | w0, w1, w2   r[sp-n] = LSE_i(r[sp-n+i] + w_i)     weighted sum
//              (LSE4: w3 in the x word of the following record)
//   LDS/LDG s               r[sp]   = slot_s   (shared / global scratch)
//   STS/STG s               slot_s  = r[sp-1]  (the next record's sp pops)
//   GLSE     | off_lo, off_hi, n   r[sp] = LSE over edge terms (slots)
//   OUT    r                out[., r] = ln2 * r[sp-1]
//   END
// Leaves: a = 1/(sigma*sqrt(2 ln 2)), b = a*mu, c = -log2(sigma*sqrt(2 pi)),
// so c - (a x - b)^2 = log2 N(x; mu, sigma).  Marginal kernels replace a leaf
// whose input is NaN by 0 (= log 1).
#pragma once
#include <stdint.h>

namespace spnb {

enum Op : uint32_t {
    OP_END = 0,
    OP_GPUSH = 1,
    OP_GACC = 2,
    OP_DPUSH = 3,
    OP_DACC = 4,
    OP_ADD = 5,
    OP_LSE1 = 6,
    OP_LSE2 = 7,
    OP_LSE3 = 8,
    OP_LSE4 = 9,
    OP_LDS = 10,
    OP_LDG = 11,
    OP_STS = 12,
    OP_STG = 13,
    OP_GLSE = 14,
    OP_OUT = 15,
    OP_NOP = 16,
    OP_COUNT = 17
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
