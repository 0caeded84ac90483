// codegen.cpp -- straight-line code for one SPN task (compiled path KS).
//
// Paper correspondence:
//   * one kernel per SPN, one sample per thread, the DAG unrolled into
//     straight-line code with constants folded in: the GPU lowering of
//     PAPER.md §IV-C (L369-382);
//   * log-space evaluation (L86): products add, weighted sums are a
//     max-shifted log-sum-exp (reading c5), here in the log2 domain with MUFU
//     ex2/lg2 and the largest input as the shift (its term is exactly 1);
//   * leaves (HiSPN Table I): Gaussian log-density, categorical /
//     histogram tables (readings c2, c3); marginal queries replace a missing
//     (NaN) leaf by log 1 = 0 (L37, L108, reading c6); NaN in a joint query
//     propagates (c7); all -inf children give -inf (c8).
//
// Pipeline: canonical DAG -> a small SSA IR of fp32 operations (this file)
// -> PTX for sm_100a (production; assembled by nvJitLink in jit.cpp, no
// C++ front end, so a 3k-node SPN compiles in about a second) and, from the
// same IR, plain C++ (used only by the CPU test-suite to check the generator
// against the oracle without a GPU).
//
// B200 specifics:
//   * Gaussian leaf on feature f, log2 N = c - (a x - b)^2 with
//     a = 1/(s sqrt(2 ln2)), b = a mu, c = -log2(s sqrt(2 pi)).  Expanded
//     around a per-feature centre M_f (x~ = x - M_f, b~ = a (mu - M_f)):
//        c - b~^2 + (2 a b~) x~ + (-a^2) x~^2
//     the constant is folded into the product's accumulator and x~, x~^2 are
//     per-sample registers, so a leaf is 2 FFMA with immediate operands and
//     no loads.  When |b~| > 8 the cancellation would cost accuracy and the
//     leaf uses the direct form t = a x~ - b~, acc -= t^2.
//   * sum weights are pushed into the children's constants ("bias"): a
//     single-parent child absorbs its parent's log2 weight (and the parent's
//     own bias) for free, so weighted sums need no adds.
//   * every node value is an SSA register; ptxas allocates registers and
//     schedules independent subtrees for ILP.
#include "codegen.h"

#include <algorithm>
#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <map>
#include <numeric>

#include "spnb.h"

namespace spnb {

namespace {

inline bool is_leaf(int32_t k) {
    return k == SPN_GAUSSIAN || k == SPN_CATEGORICAL || k == SPN_HISTOGRAM;
}

inline uint32_t fbits(float f) {
    uint32_t u;
    memcpy(&u, &f, 4);
    return u;
}

// ---------------------------------------------------------------------------
// IR: every instruction defines one fp32 SSA value (except OUT / ARGMAX).
enum IrOp {
    I_LDX,     // d = x[f]                         (aux = f)
    I_FMA,     // d = a * b + c   (round once)
    I_ADD,     // d = a + b
    I_SUB,     // d = a - b
    I_MUL,     // d = a * b
    I_MAX,     // d = max(a, b)   (NaN-ignoring)
    I_MIN,     // d = min(a, b)   (NaN-ignoring)
    I_MAXNAN,  // d = max(a, b)   (NaN-propagating)
    I_EX2,     // d = 2^a         (MUFU ex2.approx.ftz)
    I_LG2,     // d = log2(a)     (MUFU lg2.approx.ftz)
    I_SELNAN,  // d = isnan(a) ? b : c
    I_SELINF,  // d = isinf(a) ? b : c
    I_DISC,    // d = a in [lo, lo+K) ? tab[floor(a) - lo] : b;  isnan(a): joint a, marginal c
               // (log2 space: b = -inf, c = 0; linear space: b = 0, c = 1)
    I_OUT,     // out[aux] = a * ln2
    I_ARGMAX,  // argmax over out[roots] (lowest index of the largest non-NaN; -1 if none)
    I_MOV,     // d = a (immediate)
};

struct Opnd {
    int32_t reg = -1;  // >= 0: SSA value
    float imm = 0.f;   // reg < 0: immediate
};

struct Ins {
    IrOp op;
    int32_t d = -1;
    Opnd a, b, c;
    int64_t aux = 0, lo = 0, K = 0;  // I_LDX feature / I_OUT column / I_DISC table offset
};

struct Ir {
    std::vector<Ins> ins;
    int32_t nreg = 0;
    bool marg = false;
    size_t n_prologue = 0;  // leading instructions that load / prepare features
    std::vector<int32_t> argmax_roots;

    Opnd imm(double v) {
        Opnd o;
        o.imm = (float)v;
        return o;
    }
    static Opnd R(int32_t r) {
        Opnd o;
        o.reg = r;
        return o;
    }
    int32_t emit(IrOp op, Opnd a = Opnd(), Opnd b = Opnd(), Opnd c = Opnd(), int64_t aux = 0) {
        Ins i;
        i.op = op;
        i.d = nreg++;
        i.a = a;
        i.b = b;
        i.c = c;
        i.aux = aux;
        ins.push_back(i);
        return i.d;
    }
};

// Per-leaf constants (log2 domain).
struct LeafInfo {
    int32_t kind = 0, f = 0;
    double a = 0, bt = 0, c = 0;  // Gaussian
    bool expanded = true;
    int64_t tab = 0, lo = 0, K = 0;  // discrete: table offset, range [lo, lo + K)
};

constexpr double BT_MAX = 8.0;  // expanded form iff |b~| <= BT_MAX

struct FeatRegs {
    int32_t x = -1, c = -1, q = -1, d = -1, z = -1;
};

struct TaskGen {
    const CGraph &c;
    const std::vector<LeafInfo> &leaf;
    const std::vector<double> &eadd;    // explicit add per canonical edge (NaN: none)
    const std::vector<double> &pconst;  // product: bias folded into the constant
    const std::vector<double> &padd;    // product: explicit add (NaN: none)
    std::vector<FeatRegs> &fr;
    std::vector<int32_t> &val;          // SSA value per canonical node
    Ir &ir;

    double leaf_const(const LeafInfo &L) const {
        if (L.kind != SPN_GAUSSIAN) return 0.0;
        return L.expanded ? L.c - L.bt * L.bt : L.c;
    }

    // direct form: acc - t^2 with t = a x~ - b~ (t = 0 for a missing
    // feature in a marginal query, so no large constant has to cancel)
    int32_t direct_term(const LeafInfo &L, const FeatRegs &F, Opnd acc) {
        int32_t t = ir.emit(I_FMA, Ir::R(F.d), ir.imm(L.a), ir.imm(-L.bt));
        if (ir.marg) t = ir.emit(I_SELNAN, Ir::R(F.x), ir.imm(0.0), Ir::R(t));
        const int32_t nt = ir.emit(I_MUL, Ir::R(t), ir.imm(-1.0));
        return ir.emit(I_FMA, Ir::R(nt), Ir::R(t), acc);
    }

    // acc + variable part of leaf L
    int32_t leaf_terms(int32_t acc, const LeafInfo &L) {
        const FeatRegs &F = fr[L.f];
        if (L.kind == SPN_GAUSSIAN) {
            if (L.expanded) {
                acc = ir.emit(I_FMA, Ir::R(F.c), ir.imm(2.0 * L.a * L.bt), Ir::R(acc));
                acc = ir.emit(I_FMA, Ir::R(F.q), ir.imm(-L.a * L.a), Ir::R(acc));
            } else {
                acc = direct_term(L, F, Ir::R(acc));
            }
            // marginal: a missing feature has x~ = 0, x~^2 = 0 (expanded form)
            // or t = 0 (direct form), so the leaf evaluated to its constant
            // part; remove it (log 1 = 0, reading c6)
            if (ir.marg) acc = ir.emit(I_FMA, Ir::R(F.z), ir.imm(-leaf_const(L)), Ir::R(acc));
            return acc;
        }
        Ins i;
        i.op = I_DISC;
        i.d = ir.nreg++;
        i.a = Ir::R(F.x);
        i.b = ir.imm(-INFINITY);
        i.c = ir.imm(0.0);
        i.aux = L.tab;
        i.lo = L.lo;
        i.K = L.K;
        ir.ins.push_back(i);
        return ir.emit(I_ADD, Ir::R(acc), Ir::R(i.d));
    }

    // a leaf used directly as a value (sum child / root)
    int32_t inline_leaf(int64_t u, double bias) {
        const LeafInfo &L = leaf[u];
        // constant as a register-free start: (const) + terms; the first FMA
        // takes the constant as its addend
        const double k = leaf_const(L) + bias;
        if (L.kind == SPN_GAUSSIAN) {
            const FeatRegs &F = fr[L.f];
            int32_t acc;
            if (L.expanded) {
                acc = ir.emit(I_FMA, Ir::R(F.c), ir.imm(2.0 * L.a * L.bt), ir.imm(k));
                acc = ir.emit(I_FMA, Ir::R(F.q), ir.imm(-L.a * L.a), Ir::R(acc));
            } else {
                acc = direct_term(L, F, ir.imm(k));
            }
            if (ir.marg) acc = ir.emit(I_FMA, Ir::R(F.z), ir.imm(-leaf_const(L)), Ir::R(acc));
            return acc;
        }
        const int32_t z = ir.emit(I_MOV, ir.imm(k));
        return leaf_terms(z, L);
    }

    void product(int64_t u) {
        std::vector<int64_t> lv, iv;
        for (int64_t e = c.cb[u]; e < c.cb[u + 1]; ++e)
            (is_leaf(c.kind[c.ch[e]]) ? lv : iv).push_back(c.ch[e]);
        int32_t acc = -1;
        for (int64_t v : iv) acc = acc < 0 ? val[v] : ir.emit(I_ADD, Ir::R(acc), Ir::R(val[v]));
        if (!lv.empty()) {
            double k = pconst[u];
            for (int64_t l : lv) k += leaf_const(leaf[l]);
            size_t first = 0;
            if (acc >= 0) {
                if (k != 0.0) acc = ir.emit(I_ADD, Ir::R(acc), ir.imm(k));
            } else if (leaf[lv[0]].kind == SPN_GAUSSIAN) {
                // first Gaussian leaf starts from the constant (no register for it)
                acc = inline_leaf(lv[0], k - leaf_const(leaf[lv[0]]));
                first = 1;
            } else {
                acc = ir.emit(I_MOV, ir.imm(k));
            }
            for (size_t i = first; i < lv.size(); ++i) acc = leaf_terms(acc, leaf[lv[i]]);
        } else if (!std::isnan(padd[u]) && padd[u] != 0.0) {
            acc = ir.emit(I_ADD, Ir::R(acc), ir.imm(padd[u]));
        }
        val[u] = acc;
    }

    void sum(int64_t u) {
        std::vector<int32_t> t;
        for (int64_t e = c.cb[u]; e < c.cb[u + 1]; ++e) {
            const int64_t v = c.ch[e];
            if (is_leaf(c.kind[v])) t.push_back(inline_leaf(v, eadd[e]));
            else if (!std::isnan(eadd[e]) && eadd[e] != 0.0)
                t.push_back(ir.emit(I_ADD, Ir::R(val[v]), ir.imm(eadd[e])));
            else t.push_back(val[v]);
        }
        const size_t n = t.size();
        if (n == 1) {
            val[u] = t[0];
            return;
        }
        auto R = Ir::R;
        // largest input = shift (exact 1, no MUFU); the others via a min/max
        // network; hi NaN-propagating (c7); shift clamped so all -inf -> -inf (c8)
        int32_t hi;
        std::vector<int32_t> lo;
        if (n == 2) {
            hi = ir.emit(I_MAXNAN, R(t[0]), R(t[1]));
            lo.push_back(ir.emit(I_MIN, R(t[0]), R(t[1])));
        } else if (n == 3) {
            const int32_t m01 = ir.emit(I_MAX, R(t[0]), R(t[1]));
            lo.push_back(ir.emit(I_MIN, R(t[0]), R(t[1])));
            lo.push_back(ir.emit(I_MIN, R(m01), R(t[2])));
            hi = ir.emit(I_MAXNAN, R(ir.emit(I_MAXNAN, R(t[0]), R(t[1]))), R(t[2]));
        } else if (n == 4) {
            const int32_t m01 = ir.emit(I_MAX, R(t[0]), R(t[1]));
            const int32_t m23 = ir.emit(I_MAX, R(t[2]), R(t[3]));
            lo.push_back(ir.emit(I_MIN, R(t[0]), R(t[1])));
            lo.push_back(ir.emit(I_MIN, R(t[2]), R(t[3])));
            lo.push_back(ir.emit(I_MIN, R(m01), R(m23)));
            hi = ir.emit(I_MAXNAN, R(ir.emit(I_MAXNAN, R(t[0]), R(t[1]))),
                         R(ir.emit(I_MAXNAN, R(t[2]), R(t[3]))));
        } else {
            hi = t[0];
            for (size_t i = 1; i < n; ++i) hi = ir.emit(I_MAXNAN, R(hi), R(t[i]));
        }
        const int32_t hc = ir.emit(I_MAX, R(hi), ir.imm(-1e30));
        int32_t s;
        if (n <= 4) {
            s = -1;
            for (int32_t l : lo) {
                const int32_t e = ir.emit(I_EX2, R(ir.emit(I_SUB, R(l), R(hc))));
                s = s < 0 ? ir.emit(I_ADD, R(e), ir.imm(1.0)) : ir.emit(I_ADD, R(s), R(e));
            }
        } else {
            s = -1;
            for (int32_t v : t) {
                const int32_t e = ir.emit(I_EX2, R(ir.emit(I_SUB, R(v), R(hc))));
                s = s < 0 ? e : ir.emit(I_ADD, R(s), R(e));
            }
        }
        val[u] = ir.emit(I_ADD, R(hi), R(ir.emit(I_LG2, R(s))));
    }
};

// ---------------------------------------------------------------------------
// C++ back end (CPU tests): exact fp32 semantics of every IR op.
std::string cpp_opnd(const Opnd &o) {
    if (o.reg >= 0) return "r" + std::to_string(o.reg);
    char b[48];
    snprintf(b, sizeof(b), "spnb_f(0x%08xu)", fbits(o.imm));
    return b;
}

std::string emit_cpp(const Ir &ir, const std::string &fn) {
    std::string s = "static void " + fn +
                    "(const float *xr, float *o, int *am, const float *tab) {\n";
    char b[512];
    for (const Ins &i : ir.ins) {
        const std::string d = "r" + std::to_string(i.d), a = cpp_opnd(i.a), bb = cpp_opnd(i.b),
                          cc = cpp_opnd(i.c);
        switch (i.op) {
            case I_LDX: snprintf(b, sizeof(b), "const float %s = xr[%lld];", d.c_str(), (long long)i.aux); break;
            case I_MOV: snprintf(b, sizeof(b), "const float %s = %s;", d.c_str(), a.c_str()); break;
            case I_FMA: snprintf(b, sizeof(b), "const float %s = fmaf(%s, %s, %s);", d.c_str(), a.c_str(), bb.c_str(), cc.c_str()); break;
            case I_ADD: snprintf(b, sizeof(b), "const float %s = %s + %s;", d.c_str(), a.c_str(), bb.c_str()); break;
            case I_SUB: snprintf(b, sizeof(b), "const float %s = %s - %s;", d.c_str(), a.c_str(), bb.c_str()); break;
            case I_MUL: snprintf(b, sizeof(b), "const float %s = %s * %s;", d.c_str(), a.c_str(), bb.c_str()); break;
            case I_MAX: snprintf(b, sizeof(b), "const float %s = fmaxf(%s, %s);", d.c_str(), a.c_str(), bb.c_str()); break;
            case I_MIN: snprintf(b, sizeof(b), "const float %s = fminf(%s, %s);", d.c_str(), a.c_str(), bb.c_str()); break;
            case I_MAXNAN: snprintf(b, sizeof(b), "const float %s = spnb_maxn(%s, %s);", d.c_str(), a.c_str(), bb.c_str()); break;
            case I_EX2: snprintf(b, sizeof(b), "const float %s = exp2f(%s);", d.c_str(), a.c_str()); break;
            case I_LG2: snprintf(b, sizeof(b), "const float %s = log2f(%s);", d.c_str(), a.c_str()); break;
            case I_SELNAN: snprintf(b, sizeof(b), "const float %s = (%s != %s) ? %s : %s;", d.c_str(), a.c_str(), a.c_str(), bb.c_str(), cc.c_str()); break;
            case I_SELINF: snprintf(b, sizeof(b), "const float %s = (fabsf(%s) == INFINITY) ? %s : %s;", d.c_str(), a.c_str(), bb.c_str(), cc.c_str()); break;
            case I_DISC:
                snprintf(b, sizeof(b),
                         "const float %s = spnb_disc(%s, %lld, %lld, tab + %lld, %d, spnb_f(0x%08xu), "
                         "spnb_f(0x%08xu));",
                         d.c_str(), a.c_str(), (long long)i.lo, (long long)i.K, (long long)i.aux,
                         ir.marg ? 1 : 0, fbits(i.b.imm), fbits(i.c.imm));
                break;
            case I_OUT: snprintf(b, sizeof(b), "o[%lld] = %s * spnb_f(0x3f317218u);", (long long)i.aux, a.c_str()); break;
            case I_ARGMAX: {
                std::string t = "if (am) { float best = -INFINITY; int idx = -1;";
                for (int32_t r : ir.argmax_roots)
                    t += " { const float w = o[" + std::to_string(r) + "]; if (!(w != w) && (idx < 0 || w > best)) { best = w; idx = " + std::to_string(r) + "; } }";
                t += " *am = idx; }";
                snprintf(b, sizeof(b), "%s", t.substr(0, sizeof(b) - 1).c_str());
                if (t.size() >= sizeof(b)) {  // long root lists
                    s += "    " + t + "\n";
                    continue;
                }
                break;
            }
        }
        s += "    ";
        s += b;
        s += '\n';
    }
    s += "}\n";
    return s;
}

const char *kCppPrelude = R"PRE(// generated by libspnb codegen.cpp (compiled path KS, C++ back end for CPU tests)
#include <math.h>
#include <string.h>
static inline float spnb_f(unsigned u) { float f; memcpy(&f, &u, 4); return f; }
static inline float spnb_maxn(float a, float b) { return (a != a || b != b) ? NAN : (a > b ? a : b); }
static inline float spnb_disc(float x, long long lo, long long K, const float *t, int marg,
                              float outside, float missing) {
    const int ok = (x >= (float)lo) && (x < (float)(lo + K));
    float v = ok ? t[(long long)floorf(x) - lo] : outside;
    if (x != x) v = marg ? missing : x;
    return v;
}
)PRE";

// ---------------------------------------------------------------------------
// PTX back end (sm_100a).
std::string ptx_opnd(const Opnd &o, const char *pf) {
    if (o.reg >= 0) return pf + std::to_string(o.reg);
    char b[16];
    snprintf(b, sizeof(b), "0f%08X", fbits(o.imm));
    return b;
}

// Register-file prefix of sample slot j (K samples per thread interleave
// instruction by instruction: K independent copies of the body for ILP and
// K samples per instruction fetch).
const char *kSlotPrefix[4] = {"%f", "%g", "%h", "%k"};

std::string emit_ptx_entry(const Ir &ir, const std::string &name, int block, int min_blocks,
                           int K, int bar_every) {
    std::string body;
    body.reserve(ir.ins.size() * 48 * K);
    char b[4096];
    int np = 0, nr = 0, nd = 0;  // predicate / b32 / b64 temporaries
    size_t since_bar = 0;
    for (const Ins &i : ir.ins) {
      // optional CTA barrier every bar_every instructions: keeps the CTA's
      // warps in the same stretch of the straight-line body (instruction-
      // cache locality); every thread runs every iteration (see the loop)
      if (bar_every > 0 && ++since_bar >= (size_t)bar_every) {
          body += "    bar.sync 0;\n";
          since_bar = 0;
      }
      for (int j = 0; j < K; ++j) {
        const char *pf = kSlotPrefix[j];
        const std::string d = pf + std::to_string(i.d), a = ptx_opnd(i.a, pf), bb = ptx_opnd(i.b, pf),
                          cc = ptx_opnd(i.c, pf);
        const std::string xr = "%xr" + std::to_string(j), orow = "%orow" + std::to_string(j);
        switch (i.op) {
            case I_LDX: snprintf(b, sizeof(b), "ld.global.nc.f32 %s, [%s+%lld];", d.c_str(), xr.c_str(), (long long)i.aux * 4); break;
            case I_MOV: snprintf(b, sizeof(b), "mov.f32 %s, %s;", d.c_str(), a.c_str()); break;
            case I_FMA: snprintf(b, sizeof(b), "fma.rn.f32 %s, %s, %s, %s;", d.c_str(), a.c_str(), bb.c_str(), cc.c_str()); break;
            case I_ADD: snprintf(b, sizeof(b), "add.rn.f32 %s, %s, %s;", d.c_str(), a.c_str(), bb.c_str()); break;
            case I_SUB: snprintf(b, sizeof(b), "sub.rn.f32 %s, %s, %s;", d.c_str(), a.c_str(), bb.c_str()); break;
            case I_MUL: snprintf(b, sizeof(b), "mul.rn.f32 %s, %s, %s;", d.c_str(), a.c_str(), bb.c_str()); break;
            case I_MAX: snprintf(b, sizeof(b), "max.f32 %s, %s, %s;", d.c_str(), a.c_str(), bb.c_str()); break;
            case I_MIN: snprintf(b, sizeof(b), "min.f32 %s, %s, %s;", d.c_str(), a.c_str(), bb.c_str()); break;
            case I_MAXNAN: snprintf(b, sizeof(b), "max.NaN.f32 %s, %s, %s;", d.c_str(), a.c_str(), bb.c_str()); break;
            case I_EX2: snprintf(b, sizeof(b), "ex2.approx.ftz.f32 %s, %s;", d.c_str(), a.c_str()); break;
            case I_LG2: snprintf(b, sizeof(b), "lg2.approx.ftz.f32 %s, %s;", d.c_str(), a.c_str()); break;
            case I_SELNAN: {
                const int p = np++;
                snprintf(b, sizeof(b), "setp.nan.f32 %%p%d, %s, %s; selp.f32 %s, %s, %s, %%p%d;", p,
                         a.c_str(), a.c_str(), d.c_str(), bb.c_str(), cc.c_str(), p);
                break;
            }
            case I_SELINF: {
                const int p = np++;
                const std::string t = pf + std::to_string(ir.nreg + (int)(&i - ir.ins.data()));
                snprintf(b, sizeof(b), "abs.f32 %s, %s; setp.eq.f32 %%p%d, %s, 0f7F800000; selp.f32 %s, %s, %s, %%p%d;",
                         t.c_str(), a.c_str(), p, t.c_str(), d.c_str(), bb.c_str(), cc.c_str(), p);
                break;
            }
            case I_DISC: {
                char mval[16];
                snprintf(mval, sizeof(mval), "0f%08X", fbits(i.c.imm));
                const int p0 = np, r0 = nr, q0 = nd;
                np += 3;
                nr += 1;
                nd += 1;
                char lo[16], hi[16];
                snprintf(lo, sizeof(lo), "0f%08X", fbits((float)i.lo));
                snprintf(hi, sizeof(hi), "0f%08X", fbits((float)(i.lo + i.K)));
                snprintf(b, sizeof(b),
                         "setp.ge.f32 %%p%d, %s, %s; setp.lt.and.f32 %%p%d, %s, %s, %%p%d; "
                         "cvt.rmi.s32.f32 %%r%d, %s; sub.s32 %%r%d, %%r%d, %lld; "
                         "mul.wide.s32 %%rd%d, %%r%d, 4; add.s64 %%rd%d, %%tab, %%rd%d; "
                         "mov.f32 %s, 0f%08X; @%%p%d ld.global.nc.f32 %s, [%%rd%d+%lld]; "
                         "setp.nan.f32 %%p%d, %s, %s; selp.f32 %s, %s, %s, %%p%d;",
                         p0, a.c_str(), lo, p0 + 1, a.c_str(), hi, p0, r0, a.c_str(), r0, r0,
                         (long long)i.lo, q0, r0, q0, q0, d.c_str(), fbits(i.b.imm), p0 + 1,
                         d.c_str(), q0, (long long)i.aux * 4, p0 + 2, a.c_str(), a.c_str(),
                         d.c_str(), ir.marg ? mval : a.c_str(), d.c_str(), p0 + 2);
                break;
            }
            case I_OUT: {
                const std::string t = pf + std::to_string(ir.nreg + (int)(&i - ir.ins.data()));
                snprintf(b, sizeof(b), "mul.rn.f32 %s, %s, 0f3F317218; @%%pv%d st.global.f32 [%s+%lld], %s;",
                         t.c_str(), a.c_str(), j, orow.c_str(), (long long)i.aux * 4, t.c_str());
                break;
            }
            case I_ARGMAX: {
                // best / idx in registers; strict > keeps the lowest index on ties
                std::string t = "setp.ne.s64 %pam, %amp, 0; and.pred %pam, %pam, %pv" + std::to_string(j) +
                                "; @!%pam bra $Lskip_am" + std::to_string(j) +
                                "; mov.f32 %fbest, 0fFF800000; mov.s32 %ridx, -1;";
                for (int32_t r : ir.argmax_roots) {
                    char q[512];
                    snprintf(q, sizeof(q),
                             " ld.global.f32 %%fw, [%s+%d]; setp.num.f32 %%pa, %%fw, %%fw; "
                             "setp.lt.s32 %%pb, %%ridx, 0; setp.gt.or.f32 %%pb, %%fw, %%fbest, %%pb; "
                             "and.pred %%pb, %%pb, %%pa; @%%pb mov.f32 %%fbest, %%fw; @%%pb mov.s32 %%ridx, %d;",
                             orow.c_str(), r * 4, r);
                    t += q;
                }
                t += " st.global.s32 [%amrow" + std::to_string(j) + "], %ridx; $Lskip_am" + std::to_string(j) + ":";
                body += "    " + t + "\n";
                continue;
            }
        }
        body += "    ";
        body += b;
        body += '\n';
      }
    }
    // temporaries beyond the SSA values: one per I_SELINF / I_OUT instruction slot
    const int nf = ir.nreg + (int)ir.ins.size() + 1;
    std::string s;
    snprintf(b, sizeof(b),
             ".visible .entry %s(\n"
             "    .param .u64 p_x, .param .u64 p_n, .param .u64 p_ld, .param .u64 p_out,\n"
             "    .param .u32 p_R, .param .u64 p_am, .param .u64 p_tab)\n"
             ".maxntid %d, 1, 1\n"
             ".minnctapersm %d\n"
             "{\n"
             "    .reg .pred %%p<%d>;\n"
             "    .reg .pred %%pl, %%pam, %%pa, %%pb;\n"
             "    .reg .b32 %%r<%d>;\n"
             "    .reg .b64 %%rd<%d>;\n"
             "    .reg .f32 %%fbest, %%fw;\n"
             "    .reg .s32 %%ridx, %%rtid, %%rcta, %%rncta, %%R;\n"
             "    .reg .b64 %%x, %%n, %%gld, %%out, %%amp, %%tab, %%s, %%stride, %%t64, %%sj, %%sb, %%tid64;\n",
             name.c_str(), block, min_blocks, np + 1, nr + 1, nd + 1);
    s += b;
    for (int j = 0; j < K; ++j) {
        snprintf(b, sizeof(b),
                 "    .reg .f32 %s<%d>;\n"
                 "    .reg .pred %%pv%d;\n"
                 "    .reg .b64 %%xr%d, %%orow%d, %%amrow%d;\n",
                 kSlotPrefix[j], nf, j, j, j, j);
        s += b;
    }
    snprintf(b, sizeof(b),
             "    ld.param.u64 %%x, [p_x];\n"
             "    ld.param.u64 %%n, [p_n];\n"
             "    ld.param.u64 %%gld, [p_ld];\n"
             "    ld.param.u64 %%out, [p_out];\n"
             "    ld.param.u32 %%R, [p_R];\n"
             "    ld.param.u64 %%amp, [p_am];\n"
             "    ld.param.u64 %%tab, [p_tab];\n"
             "    mov.u32 %%rtid, %%tid.x;\n"
             "    mov.u32 %%rcta, %%ctaid.x;\n"
             "    mov.u32 %%rncta, %%nctaid.x;\n"
             "    mul.wide.u32 %%s, %%rcta, %d;\n"
             "    cvt.u64.u32 %%tid64, %%rtid;\n"
             "    add.s64 %%s, %%s, %%tid64;\n"
             "    mul.wide.u32 %%stride, %%rncta, %d;\n"
             "$Lloop:\n"
             "    sub.s64 %%sb, %%s, %%tid64;\n"  // CTA's first sample: the loop is CTA-uniform
             "    setp.ge.s64 %%pl, %%sb, %%n;\n"
             "    @%%pl bra $Ldone;\n",
             block * K, block * K);
    s += b;
    for (int j = 0; j < K; ++j) {
        // slot j: sample s + j*block; past the end it recomputes the CTA's
        // first sample (valid) and its stores are predicated off
        snprintf(b, sizeof(b),
                 "    add.s64 %%sj, %%s, %d;\n"
                 "    setp.lt.s64 %%pv%d, %%sj, %%n;\n"
                 "    selp.b64 %%sj, %%sj, %%sb, %%pv%d;\n"
                 "    mul.lo.s64 %%t64, %%sj, %%gld;\n"
                 "    shl.b64 %%t64, %%t64, 2;\n"
                 "    add.s64 %%xr%d, %%x, %%t64;\n"
                 "    cvt.s64.s32 %%t64, %%R;\n"
                 "    mul.lo.s64 %%t64, %%sj, %%t64;\n"
                 "    shl.b64 %%t64, %%t64, 2;\n"
                 "    add.s64 %%orow%d, %%out, %%t64;\n"
                 "    shl.b64 %%t64, %%sj, 2;\n"
                 "    add.s64 %%amrow%d, %%amp, %%t64;\n",
                 j * block, j, j, j, j, j);
        s += b;
    }
    s += body;
    s += "    add.s64 %s, %s, %stride;\n"
         "    bra $Lloop;\n"
         "$Ldone:\n"
         "    ret;\n"
         "}\n";
    return s;
}

// Largest number of simultaneously live SSA values of the inner nodes when
// the IR is executed in emission order (feature registers excluded: they are
// few and ptxas rematerialises them).  A proxy for the register pressure
// ptxas faces; straight-line code over region graphs (RAT-SPN cross
// products) reaches hundreds, where assembly time explodes.
int64_t ir_max_live(const Ir &ir) {
    std::vector<int64_t> last(ir.nreg, -1);
    std::vector<uint8_t> feat(ir.nreg, 0);
    for (size_t k = 0; k < ir.ins.size(); ++k) {
        const Ins &i = ir.ins[k];
        for (const Opnd *o : {&i.a, &i.b, &i.c})
            if (o->reg >= 0) last[o->reg] = (int64_t)k;
        if (i.d >= 0 && k < ir.n_prologue) feat[i.d] = 1;
    }
    std::vector<int32_t> dies(ir.ins.size() + 1, 0);
    for (int32_t r = 0; r < ir.nreg; ++r)
        if (!feat[r] && last[r] >= 0) dies[last[r]]++;
    int64_t live = 0, best = 0;
    for (size_t k = 0; k < ir.ins.size(); ++k) {
        const Ins &i = ir.ins[k];
        live -= dies[k];
        if (i.d >= 0 && !feat[i.d] && last[i.d] >= 0) ++live;
        best = std::max(best, live);
    }
    return best;
}

}  // namespace

int generate_jit(const GraphData &g, const JitOptions &opt, JitProgram &out, std::string &msg) {
    CGraph c;
    canonicalise(g, c);
    const int64_t n = c.n;
    out = JitProgram();

    // ---- value space (the `probability` type is chosen by
    // the compiler, e.g. from the graph depth): linear fp32 when every leaf
    // is discrete and interval bounds on the non-zero values any node can
    // take (marginalised leaves count as 1) stay inside [2^-100, 2^100] --
    // then no value can underflow or overflow fp32's normal range, sums are
    // plain FFMA chains and the only MUFU op is one lg2 per root
    {
        bool disc_only = true;
        std::vector<double> vlo(n, 1.0), vhi(n, 1.0);
        double gmin = 1.0, gmax = 1.0;
        for (int64_t u = 0; u < n && disc_only; ++u) {  // children before parents
            const int64_t o = c.orig[u];
            if (c.kind[u] == SPN_GAUSSIAN) {
                disc_only = false;
            } else if (c.kind[u] == SPN_CATEGORICAL || c.kind[u] == SPN_HISTOGRAM) {
                const double *p = g.params.data() + g.param_begin[o];
                const int64_t np = g.n_params[o];
                double lo = 1.0, hi = 1.0;  // 1: a marginalised (missing) leaf
                for (int64_t i = c.kind[u] == SPN_CATEGORICAL ? 0 : 2; i < np;
                     i += c.kind[u] == SPN_CATEGORICAL ? 1 : 3)
                    if (p[i] > 0.0) {
                        lo = std::min(lo, p[i]);
                        hi = std::max(hi, p[i]);
                    }
                vlo[u] = lo;
                vhi[u] = hi;
            } else if (c.kind[u] == SPN_PRODUCT) {
                double lo = 1.0, hi = 1.0;
                for (int64_t e = c.cb[u]; e < c.cb[u + 1]; ++e) {
                    lo *= vlo[c.ch[e]];
                    hi *= vhi[c.ch[e]];
                }
                vlo[u] = lo;
                vhi[u] = hi;
            } else {
                double lo = INFINITY, hi = 0.0;
                for (int64_t e = c.cb[u]; e < c.cb[u + 1]; ++e)
                    if (c.w[e] > 0.0) {
                        lo = std::min(lo, c.w[e] * vlo[c.ch[e]]);
                        hi += c.w[e] * vhi[c.ch[e]];
                    }
                vlo[u] = std::isfinite(lo) ? lo : 1.0;
                vhi[u] = hi > 0.0 ? hi : 1.0;
            }
            gmin = std::min(gmin, vlo[u]);
            gmax = std::max(gmax, vhi[u]);
        }
        const bool in_range = disc_only && gmin >= std::ldexp(1.0, -100) && gmax <= std::ldexp(1.0, 100);
        if (opt.space == 2 && !in_range) {
            msg = disc_only ? "linear space: value range outside [2^-100, 2^100]"
                            : "linear space needs discrete leaves only";
            return SPN_E_UNSUPPORTED;
        }
        out.linear = opt.space == 2 || (opt.space == 0 && in_range);
        out.lin_min = gmin;
        out.lin_max = gmax;
    }

    // ---- leaves: parameters in the log2 domain --------------------------
    std::vector<LeafInfo> leaf(n);
    std::vector<double> msum(g.F, 0.0);
    std::vector<int64_t> mcnt(g.F, 0);
    for (int64_t u = 0; u < n; ++u) {
        const int64_t o = c.orig[u];
        if (c.kind[u] == SPN_GAUSSIAN) {
            msum[g.feature[o]] += g.params[g.param_begin[o]];
            mcnt[g.feature[o]]++;
        }
    }
    std::vector<double> centre(g.F, 0.0);
    for (int f = 0; f < g.F; ++f)
        if (mcnt[f]) centre[f] = (double)(float)(msum[f] / (double)mcnt[f]);
    for (int64_t u = 0; u < n; ++u) {
        if (!is_leaf(c.kind[u])) continue;
        const int64_t o = c.orig[u];
        LeafInfo &L = leaf[u];
        L.kind = c.kind[u];
        L.f = g.feature[o];
        const double *p = g.params.data() + g.param_begin[o];
        const int64_t np = g.n_params[o];
        out.n_leaves++;
        if (L.kind == SPN_GAUSSIAN) {
            const double mu = p[0], sd = p[1];
            L.a = 1.0 / (sd * std::sqrt(2.0 * M_LN2));
            L.bt = L.a * (mu - centre[L.f]);
            L.c = -std::log2(sd * std::sqrt(2.0 * M_PI));
            L.expanded = std::fabs(L.bt) <= BT_MAX;
        } else if (L.kind == SPN_CATEGORICAL) {
            L.lo = 0;
            L.K = np;
            L.tab = (int64_t)out.tables.size();
            for (int64_t i = 0; i < np; ++i)
                out.tables.push_back(out.linear ? (float)p[i] : (float)std::log2(p[i]));
        } else {
            int64_t lo = INT64_MAX, hi = INT64_MIN;
            for (int64_t b = 0; b < np; b += 3) {
                lo = std::min(lo, (int64_t)p[b]);
                hi = std::max(hi, (int64_t)p[b + 1]);
            }
            std::vector<float> tab((size_t)(hi - lo), out.linear ? 0.f : -INFINITY);
            for (int64_t b = 0; b < np; b += 3)
                for (int64_t v = (int64_t)p[b]; v < (int64_t)p[b + 1]; ++v)
                    tab[v - lo] = out.linear ? (float)p[b + 2] : (float)std::log2(p[b + 2]);
            L.lo = lo;
            L.K = hi - lo;
            L.tab = (int64_t)out.tables.size();
            out.tables.insert(out.tables.end(), tab.begin(), tab.end());
        }
    }
    if (out.tables.empty()) out.tables.push_back(0.f);

    // ---- bias pushing (weights folded into the producers) ---------------
    std::vector<double> beta(n, 0.0), eadd(c.ch.size(), NAN), pconst(n, 0.0), padd(n, NAN);
    auto absorbs = [&](int64_t v) {
        return !is_leaf(c.kind[v]) && c.pb[v + 1] - c.pb[v] == 1 && c.rootrefs[v].empty();
    };
    for (int64_t u = n - 1; u >= 0; --u) {  // parents before children (post-order ids)
        if (c.kind[u] == SPN_SUM) {
            out.n_sums++;
            const int64_t fan = c.cb[u + 1] - c.cb[u];
            out.n_sum_edges += fan;
            out.mufu_per_sample += fan > 1 ? fan : 0;  // n-ary LSE: n-1 ex2 + 1 lg2
            out.mufu_exec_per_sample += fan <= 1 ? 0 : (fan <= 4 ? fan : fan + 1);
            out.fma_per_sample += 3 * fan;
            for (int64_t e = c.cb[u]; e < c.cb[u + 1]; ++e) {
                const int64_t v = c.ch[e];
                const double lw = std::log2(c.w[e]) + beta[u];
                if (!is_leaf(c.kind[v]) && absorbs(v)) beta[v] = lw;
                else eadd[e] = lw;  // leaves: folded into the inline constant
            }
        } else if (c.kind[u] == SPN_PRODUCT) {
            out.n_products++;
            bool has_leaf = false;
            int64_t first_abs = -1;
            for (int64_t e = c.cb[u]; e < c.cb[u + 1]; ++e) {
                const int64_t v = c.ch[e];
                if (is_leaf(c.kind[v])) has_leaf = true;
                else if (first_abs < 0 && absorbs(v)) first_abs = v;
                out.fma_per_sample += is_leaf(c.kind[v]) ? 0 : 1;
            }
            if (has_leaf) pconst[u] = beta[u];
            else if (first_abs >= 0) beta[first_abs] = beta[u];
            else padd[u] = beta[u];
        } else {
            out.fma_per_sample += 2;
        }
    }
    out.n_nodes = n;
    if (out.linear) {  // one lg2 per root; an FMUL per product edge, an FFMA per sum edge
        out.mufu_per_sample = out.mufu_exec_per_sample = (int64_t)g.roots.size();
        out.fma_per_sample = 0;
        for (int64_t u = 0; u < n; ++u)
            if (!is_leaf(c.kind[u])) out.fma_per_sample += c.cb[u + 1] - c.cb[u];
    }

    // ---- tasks: connected components packed up to task_cap_nodes --------
    std::vector<int64_t> uf(n);
    std::iota(uf.begin(), uf.end(), 0);
    auto find = [&](int64_t a) {
        while (uf[a] != a) a = uf[a] = uf[uf[a]];
        return a;
    };
    for (int64_t u = 0; u < n; ++u)
        for (int64_t e = c.cb[u]; e < c.cb[u + 1]; ++e) {
            const int64_t a = find(u), b = find(c.ch[e]);
            if (a != b) uf[std::max(a, b)] = std::min(a, b);
        }
    std::map<int64_t, int64_t> comp_size;
    for (int64_t u = 0; u < n; ++u) comp_size[find(u)]++;
    for (auto &kv : comp_size)
        if (kv.second > opt.max_task_nodes) {
            msg = "compiled path: connected component of " + std::to_string(kv.second) +
                  " nodes exceeds max_task_nodes " + std::to_string(opt.max_task_nodes);
            return SPN_E_UNSUPPORTED;
        }
    std::map<int64_t, int32_t> comp_task;
    std::vector<int64_t> task_size;
    for (int64_t u = 0; u < n; ++u)
        for (size_t k = 0; k < c.rootrefs[u].size(); ++k) {
            const int64_t cc = find(u);
            if (comp_task.count(cc)) continue;
            const int64_t sz = comp_size[cc];
            if (task_size.empty() || task_size.back() + sz > opt.task_cap_nodes) task_size.push_back(0);
            task_size.back() += sz;
            comp_task[cc] = (int32_t)task_size.size() - 1;
        }
    const int32_t T = (int32_t)task_size.size();
    std::vector<std::vector<int64_t>> tnodes(T);
    for (int64_t u = 0; u < n; ++u) tnodes[comp_task.at(find(u))].push_back(u);
    std::vector<std::vector<std::pair<int32_t, int64_t>>> troots(T);
    for (int64_t u = 0; u < n; ++u)
        for (int32_t r : c.rootrefs[u]) troots[comp_task.at(find(u))].push_back({r, u});
    for (auto &v : troots) std::sort(v.begin(), v.end());
    out.fused_argmax = T == 1;

    for (int32_t t = 0; t < T; ++t) {
        JitTask jt;
        jt.name = "spnb_t" + std::to_string(t);
        jt.n_nodes = (int64_t)tnodes[t].size();
        for (auto &rr : troots[t]) jt.roots.push_back(rr.first);
        std::vector<uint8_t> use_x(g.F, 0), use_c(g.F, 0), use_d(g.F, 0), use_z(g.F, 0);
        for (int64_t u : tnodes[t]) {
            if (!is_leaf(c.kind[u])) continue;
            const LeafInfo &L = leaf[u];
            use_x[L.f] = 1;
            if (L.kind == SPN_GAUSSIAN) {
                (L.expanded ? use_c : use_d)[L.f] = 1;
                use_z[L.f] = 1;
            }
        }
        std::string cpp = kCppPrelude;
        const std::string ptx_head = ".version 8.7\n.target sm_100a\n.address_size 64\n"
                                     "// generated by libspnb codegen.cpp (compiled path KS) -- do not edit\n";
        for (int marg = 0; marg < 2; ++marg) {
            Ir ir;
            ir.marg = marg != 0;
            std::vector<FeatRegs> fr(g.F);
            std::vector<int32_t> val(n, -1);
            TaskGen tg{c, leaf, eadd, pconst, padd, fr, val, ir};
            auto R = Ir::R;
            for (int f = 0; f < g.F; ++f) {
                if (!use_x[f]) continue;
                FeatRegs &F = fr[f];
                F.x = ir.emit(I_LDX, Opnd(), Opnd(), Opnd(), f);
                const bool has_m = centre[f] != 0.0;
                const int32_t xm = (use_c[f] || use_d[f]) && has_m
                                       ? ir.emit(I_SUB, R(F.x), ir.imm(centre[f]))
                                       : F.x;
                if (ir.marg && use_z[f]) F.z = ir.emit(I_SELNAN, R(F.x), ir.imm(1.0), ir.imm(0.0));
                if (use_c[f]) {
                    // x~ and x~^2; an infinite input gives x~ = 0 and x~^2 = inf,
                    // so the leaf is -inf (not inf - inf)
                    const int32_t c0 = ir.marg ? ir.emit(I_SELNAN, R(F.x), ir.imm(0.0), R(xm)) : xm;
                    F.q = ir.emit(I_MUL, R(c0), R(c0));
                    F.c = ir.emit(I_SELINF, R(F.x), ir.imm(0.0), R(c0));
                }
                if (use_d[f]) F.d = ir.marg ? ir.emit(I_SELNAN, R(F.x), ir.imm(0.0), R(xm)) : xm;
            }
            ir.n_prologue = ir.ins.size();
            if (out.linear) {
                // linear space: leaf = p (0 outside the support, 1 if missing
                // in a marginal query); product = FMUL chain; sum = FFMA chain
                // with the weights as immediates
                for (int64_t u : tnodes[t]) {
                    if (is_leaf(c.kind[u])) {
                        const LeafInfo &L = leaf[u];
                        Ins i;
                        i.op = I_DISC;
                        i.d = ir.nreg++;
                        i.a = R(fr[L.f].x);
                        i.b = ir.imm(0.0);
                        i.c = ir.imm(1.0);
                        i.aux = L.tab;
                        i.lo = L.lo;
                        i.K = L.K;
                        ir.ins.push_back(i);
                        val[u] = i.d;
                    } else if (c.kind[u] == SPN_PRODUCT) {
                        int32_t acc = val[c.ch[c.cb[u]]];
                        for (int64_t e = c.cb[u] + 1; e < c.cb[u + 1]; ++e)
                            acc = ir.emit(I_MUL, R(acc), R(val[c.ch[e]]));
                        val[u] = acc;
                    } else {
                        int32_t acc = ir.emit(I_MUL, R(val[c.ch[c.cb[u]]]), ir.imm(c.w[c.cb[u]]));
                        for (int64_t e = c.cb[u] + 1; e < c.cb[u + 1]; ++e)
                            acc = ir.emit(I_FMA, R(val[c.ch[e]]), ir.imm(c.w[e]), R(acc));
                        val[u] = acc;
                    }
                }
            } else {
                for (int64_t u : tnodes[t]) {
                    if (c.kind[u] == SPN_PRODUCT) tg.product(u);
                    else if (c.kind[u] == SPN_SUM) tg.sum(u);
                }
            }
            for (auto &rr : troots[t]) {
                const int64_t u = rr.second;
                int32_t v;
                if (out.linear) v = ir.emit(I_LG2, R(val[u]));
                else v = is_leaf(c.kind[u]) ? tg.inline_leaf(u, 0.0) : val[u];
                Ins o;
                o.op = I_OUT;
                o.a = R(v);
                o.aux = rr.first;
                ir.ins.push_back(o);
            }
            if (out.fused_argmax) {
                Ins a;
                a.op = I_ARGMAX;
                ir.argmax_roots = jt.roots;
                ir.ins.push_back(a);
            }
            const std::string suffix = marg ? "_m" : "_j";
            jt.max_live = std::max(jt.max_live, ir_max_live(ir));
            if (getenv("SPNB_JIT_VERBOSE"))
                fprintf(stderr, "[spnb] task %d marg %d: %zu ins, max_live %lld\n", t, marg, ir.ins.size(),
                        (long long)ir_max_live(ir));
            jt.ptx[marg] = ptx_head + emit_ptx_entry(ir, jt.name + suffix, opt.block, opt.min_blocks,
                                                       opt.samples_per_thread, opt.bar_every);
            cpp += emit_cpp(ir, jt.name + suffix + "_body");
        }
        char b[1024];
        snprintf(b, sizeof(b),
                 "extern \"C\" void %s_host(const float *x, long long n, long long ld, float *out, int R, "
                 "int *argmax, const float *tab, int marg) {\n"
                 "  for (long long s = 0; s < n; ++s) {\n"
                 "    if (marg) %s_m_body(x + s * ld, out + s * R, argmax ? argmax + s : 0, tab);\n"
                 "    else %s_j_body(x + s * ld, out + s * R, argmax ? argmax + s : 0, tab);\n"
                 "  }\n"
                 "}\n",
                 jt.name.c_str(), jt.name.c_str(), jt.name.c_str());
        cpp += b;
        jt.source = jt.ptx[0] + jt.ptx[1];
        jt.cpp = std::move(cpp);
        int64_t nf = 0;
        for (int f = 0; f < g.F; ++f) nf += use_x[f];
        jt.n_features = nf;
        out.tasks.push_back(std::move(jt));
    }
    return SPN_OK;
}

}  // namespace spnb
