// dag_eval.cuh -- generic SPN DAG evaluator for sm_100a (kernel KA).
//
// Computes, for every sample s and root r, log p_r(x_s) by a single bottom-up
// pass over the DAG (§II-A): leaves query univariate
// distributions with full (joint) or partial (marginal) evidence, products add
// log values, weighted sums take a max-shifted log-sum-exp (log space, L86).
//
// B200 design:
//  * The DAG is not compiled to straight-line code per SPN as in the paper's
//    GPU lowering (L369-382); it is a table-driven node program (program.h)
//    interpreted by every thread for K samples at once, so one warp-uniform
//    dispatch is amortised over 32*K samples.  Values live in a register
//    stack whose depth at each record is static: one dense switch with a case
//    per (op, sp) compiles to a single jump table (LDC + BRX).
//  * Each warp owns a tile of 32*K samples; the tile's features are staged in
//    shared memory transposed to [F][32K+4] so a leaf reads its K inputs with
//    one vector LDS (the paper's access-pattern-aware loads, L80, L360).
//  * Sums use the n-ary max-shifted LSE in the log2 domain with MUFU ex2/lg2:
//    fan-in + 1 MUFU ops per sum (not 2 per edge as binary log-adds).
//  * Single-task plans: the node program is staged once per CTA and warps run
//    a persistent static round-robin loop over warp tiles (no CTA barriers).
//    Multi-task plans (partitioned, L336-346): CTA tiles, each task's program
//    is staged into shared memory in turn; values crossing tasks go through
//    per-warp global scratch slots (L2 resident), task-local ones through
//    shared-memory slots.
#pragma once
#include <cuda_runtime.h>
#include <math_constants.h>
#include <stdint.h>

#include "program.h"

namespace spnb {

__device__ __forceinline__ float ex2a(float x) {
    float y;
    asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
    return y;
}
__device__ __forceinline__ float lg2a(float x) {
    float y;
    asm("lg2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
    return y;
}

__device__ __forceinline__ Rec make_end() {
    Rec r;
    r.x = 0; r.y = 0; r.z = 0; r.w = 0;
    return r;
}

// 32-bit shared-memory addressing through asm: the addresses are "pinned" in
// registers (a volatile mov cannot be rematerialised), so the compiler does not
// recompute the warp's tile base in every switch case.
__device__ __forceinline__ uint32_t pin_u32(uint32_t v) {
    uint32_t r;
    asm volatile("mov.b32 %0, %1;" : "=r"(r) : "r"(v));
    return r;
}
__device__ __forceinline__ uint32_t smem_u32(const void *p) {
    return (uint32_t)__cvta_generic_to_shared(p);
}

template <int K>
struct SIO;  // shared memory, 32-bit byte address
template <>
struct SIO<4> {
    static __device__ __forceinline__ void ld(uint32_t a, float (&v)[4]) {
        asm volatile("ld.shared.v4.f32 {%0, %1, %2, %3}, [%4];"
                     : "=f"(v[0]), "=f"(v[1]), "=f"(v[2]), "=f"(v[3]) : "r"(a));
    }
    static __device__ __forceinline__ void st(uint32_t a, const float (&v)[4]) {
        asm volatile("st.shared.v4.f32 [%0], {%1, %2, %3, %4};"
                     :: "r"(a), "f"(v[0]), "f"(v[1]), "f"(v[2]), "f"(v[3]) : "memory");
    }
};
template <>
struct SIO<8> {
    static __device__ __forceinline__ void ld(uint32_t a, float (&v)[8]) {
        asm volatile("ld.shared.v4.f32 {%0, %1, %2, %3}, [%4];"
                     : "=f"(v[0]), "=f"(v[1]), "=f"(v[2]), "=f"(v[3]) : "r"(a));
        asm volatile("ld.shared.v4.f32 {%0, %1, %2, %3}, [%4];"
                     : "=f"(v[4]), "=f"(v[5]), "=f"(v[6]), "=f"(v[7]) : "r"(a + 16));
    }
    static __device__ __forceinline__ void st(uint32_t a, const float (&v)[8]) {
        asm volatile("st.shared.v4.f32 [%0], {%1, %2, %3, %4};"
                     :: "r"(a), "f"(v[0]), "f"(v[1]), "f"(v[2]), "f"(v[3]) : "memory");
        asm volatile("st.shared.v4.f32 [%0], {%1, %2, %3, %4};"
                     :: "r"(a + 16), "f"(v[4]), "f"(v[5]), "f"(v[6]), "f"(v[7]) : "memory");
    }
};
template <>
struct SIO<2> {
    static __device__ __forceinline__ void ld(uint32_t a, float (&v)[2]) {
        asm volatile("ld.shared.v2.f32 {%0, %1}, [%2];" : "=f"(v[0]), "=f"(v[1]) : "r"(a));
    }
    static __device__ __forceinline__ void st(uint32_t a, const float (&v)[2]) {
        asm volatile("st.shared.v2.f32 [%0], {%1, %2};" :: "r"(a), "f"(v[0]), "f"(v[1])
                     : "memory");
    }
};
template <>
struct SIO<1> {
    static __device__ __forceinline__ void ld(uint32_t a, float (&v)[1]) {
        asm volatile("ld.shared.f32 %0, [%1];" : "=f"(v[0]) : "r"(a));
    }
    static __device__ __forceinline__ void st(uint32_t a, const float (&v)[1]) {
        asm volatile("st.shared.f32 [%0], %1;" :: "r"(a), "f"(v[0]) : "memory");
    }
};

template <int K>
struct GIO;  // global memory (scratch slots)
template <>
struct GIO<4> {
    static __device__ __forceinline__ void ld(const float *p, float (&v)[4]) {
        const float4 t = *reinterpret_cast<const float4 *>(p);
        v[0] = t.x; v[1] = t.y; v[2] = t.z; v[3] = t.w;
    }
    static __device__ __forceinline__ void st(float *p, const float (&v)[4]) {
        *reinterpret_cast<float4 *>(p) = make_float4(v[0], v[1], v[2], v[3]);
    }
};
template <>
struct GIO<8> {
    static __device__ __forceinline__ void ld(const float *p, float (&v)[8]) {
        const float4 t = *reinterpret_cast<const float4 *>(p);
        const float4 u = *reinterpret_cast<const float4 *>(p + 4);
        v[0] = t.x; v[1] = t.y; v[2] = t.z; v[3] = t.w;
        v[4] = u.x; v[5] = u.y; v[6] = u.z; v[7] = u.w;
    }
    static __device__ __forceinline__ void st(float *p, const float (&v)[8]) {
        *reinterpret_cast<float4 *>(p) = make_float4(v[0], v[1], v[2], v[3]);
        *reinterpret_cast<float4 *>(p + 4) = make_float4(v[4], v[5], v[6], v[7]);
    }
};
template <>
struct GIO<2> {
    static __device__ __forceinline__ void ld(const float *p, float (&v)[2]) {
        const float2 t = *reinterpret_cast<const float2 *>(p);
        v[0] = t.x; v[1] = t.y;
    }
    static __device__ __forceinline__ void st(float *p, const float (&v)[2]) {
        *reinterpret_cast<float2 *>(p) = make_float2(v[0], v[1]);
    }
};
template <>
struct GIO<1> {
    static __device__ __forceinline__ void ld(const float *p, float (&v)[1]) { v[0] = *p; }
    static __device__ __forceinline__ void st(float *p, const float (&v)[1]) { *p = v[0]; }
};

// Per-thread execution environment.  Record operands for features and slots
// are BYTE offsets (pre-multiplied by the preparer).
template <int K, bool MARG, bool XS>
struct Env {
    uint32_t xs;            // XS: shared address of this thread's x column (+lane*K*4)
    const float *xrow[K];   // !XS: row pointers of this thread's K samples
    uint32_t ss;            // shared slots of this warp (+lane*K*4)
    char *gs;               // global slots of this warp (+lane*K*4)
    const float *tables;
    const Edge *edges;
    float *out;             // out + first sample * R
    int32_t R;
    int32_t nvalid;         // valid samples of this thread (0..K)

    __device__ __forceinline__ void loadx(uint32_t f, float (&v)[K]) const {
        if constexpr (XS) {
            SIO<K>::ld(xs + f, v);
        } else {
#pragma unroll
            for (int j = 0; j < K; ++j)
                v[j] = __ldg(reinterpret_cast<const float *>(
                    reinterpret_cast<const char *>(xrow[j]) + f));
        }
    }
    __device__ __forceinline__ void load_slot(uint32_t ref, float (&v)[K]) const {
        if (ref & SLOT_GLOBAL) GIO<K>::ld(reinterpret_cast<const float *>(gs + (ref & ~SLOT_GLOBAL)), v);
        else SIO<K>::ld(ss + ref, v);
    }
};

#define FOR_K _Pragma("unroll") for (int j = 0; j < K; ++j)

__device__ __forceinline__ void lds4(uint32_t a, uint32_t &x, uint32_t &y, uint32_t &z,
                                     uint32_t &w) {
    asm volatile("ld.shared.v4.u32 {%0, %1, %2, %3}, [%4];"
                 : "=r"(x), "=r"(y), "=r"(z), "=r"(w) : "r"(a));
}

// Leaf product: acc = C + sum_i leaf_i over the parameter records at pp
// (ng Gaussian then nd discrete).  Returns the address after the last one.
template <int S, bool ACC, int D, int K, bool MARG, bool XS>
__device__ __forceinline__ uint32_t h_lprod(float (&r)[D][K], uint32_t ng, float C,
                                            uint32_t nd, uint32_t pp,
                                            const Env<K, MARG, XS> &e) {
    float acc[K];
    if constexpr (ACC) {
        FOR_K acc[j] = r[S - 1][j] + C;
    } else {
        FOR_K acc[j] = C;
    }
#pragma unroll 2
    for (uint32_t i = 0; i < ng; ++i, pp += 16) {
        uint32_t f, ya, zb, wc;
        lds4(pp, f, ya, zb, wc);
        float xv[K];
        e.loadx(f, xv);
        const float a = __uint_as_float(ya), b = __uint_as_float(zb);
        FOR_K {
            const float t = fmaf(a, xv[j], -b);
            if constexpr (MARG) {
                // NaN input: subtract this leaf's c from the pre-summed C instead
                // of t^2, i.e. the leaf contributes log 1 = 0 (reading c6)
                const bool nan = xv[j] != xv[j];
                const float pv = nan ? __uint_as_float(wc) : t;
                const float qv = nan ? 1.f : t;
                acc[j] = fmaf(-pv, qv, acc[j]);
            } else {
                acc[j] = fmaf(-t, t, acc[j]);
            }
        }
    }
    for (uint32_t i = 0; i < nd; ++i, pp += 16) {
        uint32_t f, tb, lo_u, nk;
        lds4(pp, f, tb, lo_u, nk);
        float xv[K];
        e.loadx(f, xv);
        const float *tab = e.tables + tb;
        const int lo = (int)lo_u;
        const float flo = (float)lo, fhi = (float)(lo + (int)nk);
        FOR_K {
            const float x = xv[j];
            const bool ok = (x >= flo) && (x < fhi);
            const int idx = ok ? ((int)floorf(x) - lo) : 0;
            float v = ok ? __ldg(tab + idx) : -CUDART_INF_F;
            if (x != x) v = MARG ? 0.f : x;
            acc[j] += v;
        }
    }
    if constexpr (ACC) {
        FOR_K r[S - 1][j] = acc[j];
    } else {
        FOR_K r[S][j] = acc[j];
    }
    return pp;
}

__device__ __forceinline__ float max_nan(float a, float b) {  // NaN-propagating max
    float r;
    asm("max.NaN.f32 %0, %1, %2;" : "=f"(r) : "f"(a), "f"(b));
    return r;
}

// n-ary max-shifted log-sum-exp in the log2 domain.  The largest input hi is
// the shift, so its term ex2(0) = 1 is exact and needs no MUFU: the n-1 other
// inputs (selected with a min/max network) cost one ex2 each, plus one lg2.
//   r = hi + bias + lg2(1 + sum_i ex2(lo_i - hi))
// hi is NaN-propagating (reading c7); with all inputs -inf the shift is
// clamped so the result is -inf, not NaN (reading c8).
template <int N>
__device__ __forceinline__ float lse_vals(const float (&v)[N], float bias) {
    float hi, lo[N - 1];
    if constexpr (N == 2) {
        hi = max_nan(v[0], v[1]);
        lo[0] = fminf(v[0], v[1]);
    } else if constexpr (N == 3) {
        const float m01 = fmaxf(v[0], v[1]);
        lo[0] = fminf(v[0], v[1]);
        lo[1] = fminf(m01, v[2]);
        hi = max_nan(max_nan(v[0], v[1]), v[2]);
    } else {
        const float m01 = fmaxf(v[0], v[1]), m23 = fmaxf(v[2], v[3]);
        lo[0] = fminf(v[0], v[1]);
        lo[1] = fminf(v[2], v[3]);
        lo[2] = fminf(m01, m23);
        hi = max_nan(max_nan(v[0], v[1]), max_nan(v[2], v[3]));
    }
    const float hc = fmaxf(hi, -1e30f);
    float s = 1.f;
#pragma unroll
    for (int i = 0; i < N - 1; ++i) s += ex2a(lo[i] - hc);
    return (hi + bias) + lg2a(s);
}

template <int S, int N, int D, int K>
__device__ __forceinline__ void h_lse(float (&r)[D][K], float bias) {
    FOR_K {
        if constexpr (N == 1) {
            r[S - 1][j] += bias;
        } else {
            float v[N];
#pragma unroll
            for (int i = 0; i < N; ++i) v[i] = r[S - N + i][j];
            r[S - N][j] = lse_vals<N>(v, bias);
        }
    }
}

// One Gaussian leaf (parameter record at pp) accumulated into acc.
template <int K, bool MARG, bool XS>
__device__ __forceinline__ void gauss_acc(float (&acc)[K], uint32_t pp, const Env<K, MARG, XS> &e) {
    uint32_t f, ya, zb, wc;
    lds4(pp, f, ya, zb, wc);
    float xv[K];
    e.loadx(f, xv);
    const float a = __uint_as_float(ya), b = __uint_as_float(zb);
    FOR_K {
        const float t = fmaf(a, xv[j], -b);
        if constexpr (MARG) {
            const bool nan = xv[j] != xv[j];
            const float pv = nan ? __uint_as_float(wc) : t;
            const float qv = nan ? 1.f : t;
            acc[j] = fmaf(-pv, qv, acc[j]);
        } else {
            acc[j] = fmaf(-t, t, acc[j]);
        }
    }
}

// Fused weighted sum over KC Gaussian leaf products (SLPk record).
template <int S, int KC, int D, int K, bool MARG, bool XS>
__device__ __forceinline__ void h_slp(float (&r)[D][K], uint32_t counts, float bias,
                                      const float (&Cs)[4], uint32_t pp,
                                      const Env<K, MARG, XS> &e) {
    float v[KC][K];
#pragma unroll
    for (int c = 0; c < KC; ++c) {
        const uint32_t nc = (counts >> (3 * c)) & 7u;
        float acc[K];
        FOR_K acc[j] = Cs[c];
#pragma unroll 1
        for (uint32_t i = 0; i < nc; ++i, pp += 16) gauss_acc<K, MARG, XS>(acc, pp, e);
        FOR_K v[c][j] = acc[j];
    }
    FOR_K {
        float w[KC];
#pragma unroll
        for (int c = 0; c < KC; ++c) w[c] = v[c][j];
        r[S][j] = lse_vals<KC>(w, bias);
    }
}

// Straight-line fused sum over KC children of 2 Gaussian leaves each.
template <int S, int KC, int D, int K, bool MARG, bool XS>
__device__ __forceinline__ void h_slpu(float (&r)[D][K], float bias, const float (&Cs)[4],
                                       const uint32_t (&fo)[6], uint32_t pp,
                                       const Env<K, MARG, XS> &e) {
    constexpr int NL = 2 * KC;
    float xv[NL][K];
#pragma unroll
    for (int i = 0; i < NL; ++i) e.loadx(fo[i], xv[i]);
    uint32_t f[NL], ya[NL], zb[NL], wc[NL];
#pragma unroll
    for (int i = 0; i < NL; ++i) lds4(pp + 16 * i, f[i], ya[i], zb[i], wc[i]);
    float v[KC][K];
#pragma unroll
    for (int c = 0; c < KC; ++c) {
        FOR_K v[c][j] = Cs[c];
#pragma unroll
        for (int l = 0; l < 2; ++l) {
            const int i = 2 * c + l;
            const float a = __uint_as_float(ya[i]), b = __uint_as_float(zb[i]);
            FOR_K {
                const float t = fmaf(a, xv[i][j], -b);
                if constexpr (MARG) {
                    const bool nan = xv[i][j] != xv[i][j];
                    v[c][j] = fmaf(-(nan ? __uint_as_float(wc[i]) : t), nan ? 1.f : t, v[c][j]);
                } else {
                    v[c][j] = fmaf(-t, t, v[c][j]);
                }
            }
        }
    }
    FOR_K {
        float w[KC];
#pragma unroll
        for (int c = 0; c < KC; ++c) w[c] = v[c][j];
        r[S][j] = lse_vals<KC>(w, bias);
    }
}

// Straight-line product of exactly N Gaussian leaves.  The header carries the
// leaves' feature offsets (16 bits each, fo), so the feature loads are issued
// together with the parameter loads (records at pp: {-, a, b, c}).
template <int S, bool ACC, int N, int D, int K, bool MARG, bool XS>
__device__ __forceinline__ void h_gprod(float (&r)[D][K], float C, uint32_t fo01, uint32_t fo23,
                                        uint32_t pp, const Env<K, MARG, XS> &e) {
    const uint32_t fo[4] = {fo01 & 0xffffu, fo01 >> 16, fo23 & 0xffffu, fo23 >> 16};
    float xv[N][K];
#pragma unroll
    for (int i = 0; i < N; ++i) e.loadx(fo[i], xv[i]);
    uint32_t f[N], ya[N], zb[N], wc[N];
#pragma unroll
    for (int i = 0; i < N; ++i) lds4(pp + 16 * i, f[i], ya[i], zb[i], wc[i]);
    float acc[K];
    if constexpr (ACC) {
        FOR_K acc[j] = r[S - 1][j] + C;
    } else {
        FOR_K acc[j] = C;
    }
#pragma unroll
    for (int i = 0; i < N; ++i) {
        const float a = __uint_as_float(ya[i]), b = __uint_as_float(zb[i]);
        FOR_K {
            const float t = fmaf(a, xv[i][j], -b);
            if constexpr (MARG) {
                const bool nan = xv[i][j] != xv[i][j];
                const float pv = nan ? __uint_as_float(wc[i]) : t;
                const float qv = nan ? 1.f : t;
                acc[j] = fmaf(-pv, qv, acc[j]);
            } else {
                acc[j] = fmaf(-t, t, acc[j]);
            }
        }
    }
    if constexpr (ACC) {
        FOR_K r[S - 1][j] = acc[j];
    } else {
        FOR_K r[S][j] = acc[j];
    }
}

template <int K>
struct VecK {
    float v[K];
};

// Gather-LSE over slot terms (large fan-in sums whose children are stored).
// Not inlined: one copy serves every stack depth; arguments and result are
// passed by value so the caller's register stack stays in registers.
template <int K>
__device__ __noinline__ VecK<K> h_glse(const Edge *__restrict__ E, int n, uint32_t ss,
                                      const char *gs) {
    auto load = [&](uint32_t ref, float (&v)[K]) {
        if (ref & SLOT_GLOBAL) GIO<K>::ld(reinterpret_cast<const float *>(gs + (ref & ~SLOT_GLOBAL)), v);
        else SIO<K>::ld(ss + ref, v);
    };
    float m[K];
    FOR_K m[j] = -CUDART_INF_F;
    for (int i = 0; i < n; ++i) {
        const Edge ed = E[i];
        float v[K];
        load(ed.a, v);
        if (ed.b != SLOT_NONE) {
            float u[K];
            load(ed.b, u);
            FOR_K v[j] += u[j];
        }
        FOR_K m[j] = fmaxf(m[j], v[j] + ed.lw);
    }
    float s[K];
    FOR_K {
        m[j] = fmaxf(m[j], -1e30f);
        s[j] = 0.f;
    }
    for (int i = 0; i < n; ++i) {
        const Edge ed = E[i];
        float v[K];
        load(ed.a, v);
        if (ed.b != SLOT_NONE) {
            float u[K];
            load(ed.b, u);
            FOR_K v[j] += u[j];
        }
        FOR_K s[j] += ex2a(v[j] + ed.lw - m[j]);
    }
    VecK<K> out;
    FOR_K out.v[j] = m[j] + lg2a(s[j]);
    return out;
}

template <int K>
struct ArgState {
    float best[K];
    int32_t idx[K];
    __device__ __forceinline__ void init() {
        FOR_K {
            best[j] = -CUDART_INF_F;
            idx[j] = -1;
        }
    }
};

template <int S, int D, int K, bool MARG, bool XS>
__device__ __forceinline__ void h_out(float (&r)[D][K], uint32_t root,
                                      const Env<K, MARG, XS> &e, ArgState<K> &am) {
    FOR_K {
        const float v = r[S - 1][j] * 0.6931471805599453f;
        if (j < e.nvalid) e.out[j * e.R + (int)root] = v;
        if (!(v != v) && (am.idx[j] < 0 || v > am.best[j] ||
                          (v == am.best[j] && (int)root < am.idx[j]))) {
            am.best[j] = v;
            am.idx[j] = (int)root;
        }
    }
}

// ---------------------------------------------------------------------------
// Valid stack depths per op (sp = depth before the op).
__host__ __device__ constexpr bool op_valid(int op, int sp, int D) {
    if (sp > D) return false;
    return (op == OP_LPUSH || op == OP_LDS || op == OP_LDG || op == OP_GLSE ||
            (op >= OP_GPUSH1 && op <= OP_GPUSH4) || (op >= OP_SLP2 && op <= OP_SLP4) ||
            op == OP_SLPU2 || op == OP_SLPU3)
               ? (sp >= 0 && sp < D)
           : (op == OP_LACC || op == OP_LSE1 || op == OP_STS || op == OP_STG || op == OP_OUT ||
              (op >= OP_GACC1 && op <= OP_GACC4))
               ? (sp >= 1)
           : (op == OP_ADD || op == OP_LSE2) ? (sp >= 2)
           : (op == OP_LSE3) ? (sp >= 3)
           : (op == OP_LSE4) ? (sp >= 4)
           : (op == OP_NOP);
}

#define SPN_ALL_SP(M, O) M(O, 0) M(O, 1) M(O, 2) M(O, 3) M(O, 4) M(O, 5) M(O, 6) M(O, 7) \
    M(O, 8) M(O, 9) M(O, 10) M(O, 11) M(O, 12) M(O, 13) M(O, 14) M(O, 15) M(O, 16)

// Every case label op*17+sp exists (dense => one jump table); invalid
// combinations end the task.
#define SPN_CASE(O, S)                                                           \
    case O * NSP + S:                                                            \
        if constexpr (op_valid(O, S, D)) {                                          \
            SPN_BODY_##O(S)                                                      \
        } else {                                                                 \
            return;                                                              \
        }                                                                        \
        break;

#define SPN_BODY_0(S) ;
// Every body captures its operands, advances pc, issues the load of the next
// record into (cx, cy, cz, cw) -- so its latency overlaps the body -- and then
// computes.
#define SPN_NEXT(NEWPC)                                                          \
    pc = (NEWPC);                                                                \
    lds4(pc, cx, cy, cz, cw);
#define SPN_SS(S) (S < D ? S : 0)
#define SPN_BODY_1(S)                                                            \
    {                                                                            \
        const uint32_t ng = cx >> CASE_BITS, nd = cz, pp = pc + 16;              \
        const float C = __uint_as_float(cy);                                     \
        SPN_NEXT(pc + 16 * (1 + ng + nd))                                        \
        h_lprod<SPN_SS(S), false>(r, ng, C, nd, pp, e);                          \
    }
#define SPN_BODY_2(S)                                                            \
    {                                                                            \
        const uint32_t ng = cx >> CASE_BITS, nd = cz, pp = pc + 16;              \
        const float C = __uint_as_float(cy);                                     \
        SPN_NEXT(pc + 16 * (1 + ng + nd))                                        \
        h_lprod<S, true>(r, ng, C, nd, pp, e);                                   \
    }
#define SPN_BODY_3(S)                                                            \
    {                                                                            \
        const float b = __uint_as_float(cy);                                     \
        SPN_NEXT(pc + 16)                                                        \
        FOR_K r[S - 2][j] += r[S - 1][j] + b;                                    \
    }
#define SPN_LSE_BODY(S, N)                                                       \
    {                                                                            \
        const float b = __uint_as_float(cy);                                     \
        SPN_NEXT(pc + 16)                                                        \
        h_lse<S, N>(r, b);                                                       \
    }
#define SPN_BODY_4(S) SPN_LSE_BODY(S, 1)
#define SPN_BODY_5(S) SPN_LSE_BODY(S, 2)
#define SPN_BODY_6(S) SPN_LSE_BODY(S, 3)
#define SPN_BODY_7(S) SPN_LSE_BODY(S, 4)
#define SPN_BODY_8(S)                                                            \
    {                                                                            \
        const uint32_t a = cx >> CASE_BITS;                                      \
        const float b = __uint_as_float(cy);                                     \
        SPN_NEXT(pc + 16)                                                        \
        SIO<K>::ld(e.ss + a, r[SPN_SS(S)]);                                      \
        FOR_K r[SPN_SS(S)][j] += b;                                              \
    }
#define SPN_BODY_9(S)                                                            \
    {                                                                            \
        const uint32_t a = cz; /* global slot byte offset (32 bits) */           \
        const float b = __uint_as_float(cy);                                     \
        SPN_NEXT(pc + 16)                                                        \
        GIO<K>::ld(reinterpret_cast<const float *>(e.gs + a), r[SPN_SS(S)]);     \
        FOR_K r[SPN_SS(S)][j] += b;                                              \
    }
#define SPN_BODY_10(S)                                                           \
    {                                                                            \
        const uint32_t a = cx >> CASE_BITS;                                      \
        SPN_NEXT(pc + 16)                                                        \
        SIO<K>::st(e.ss + a, r[S - 1]);                                          \
    }
#define SPN_BODY_11(S)                                                           \
    {                                                                            \
        const uint32_t a = cz; /* global slot byte offset (32 bits) */           \
        SPN_NEXT(pc + 16)                                                        \
        GIO<K>::st(reinterpret_cast<float *>(e.gs + a), r[S - 1]);               \
    }
#define SPN_BODY_12(S)                                                           \
    {                                                                            \
        const Edge *E = e.edges + (((uint64_t)cz << 32) | cy);                   \
        const int n = (int)cw;                                                   \
        SPN_NEXT(pc + 16)                                                        \
        const VecK<K> g = h_glse<K>(E, n, e.ss, e.gs);                           \
        FOR_K r[SPN_SS(S)][j] = g.v[j];                                          \
    }
#define SPN_BODY_13(S)                                                           \
    {                                                                            \
        const uint32_t root = cx >> CASE_BITS;                                   \
        SPN_NEXT(pc + 16)                                                        \
        h_out<S>(r, root, e, am);                                                \
    }
#define SPN_BODY_14(S) SPN_NEXT(pc + 16)
#define SPN_GPROD_BODY(S, ACC, N)                                                \
    {                                                                            \
        const float C = __uint_as_float(cy);                                     \
        const uint32_t fo01 = cz, fo23 = cw, pp = pc + 16;                       \
        SPN_NEXT(pc + 16 * (N + 1))                                              \
        h_gprod<S, ACC, N>(r, C, fo01, fo23, pp, e);                             \
    }
#define SPN_BODY_15(S) SPN_GPROD_BODY(SPN_SS(S), false, 1)
#define SPN_BODY_16(S) SPN_GPROD_BODY(SPN_SS(S), false, 2)
#define SPN_BODY_17(S) SPN_GPROD_BODY(SPN_SS(S), false, 3)
#define SPN_BODY_18(S) SPN_GPROD_BODY(SPN_SS(S), false, 4)
#define SPN_BODY_19(S) SPN_GPROD_BODY(S, true, 1)
#define SPN_BODY_20(S) SPN_GPROD_BODY(S, true, 2)
#define SPN_BODY_21(S) SPN_GPROD_BODY(S, true, 3)
#define SPN_BODY_22(S) SPN_GPROD_BODY(S, true, 4)
#define SPN_SLP_BODY(S, KC)                                                      \
    {                                                                            \
        const uint32_t counts = cx >> CASE_BITS;                                 \
        float Cs[4];                                                             \
        Cs[0] = __uint_as_float(cz);                                             \
        Cs[1] = __uint_as_float(cw);                                             \
        Cs[2] = 0.f;                                                             \
        Cs[3] = 0.f;                                                             \
        const float bias = __uint_as_float(cy);                                  \
        uint32_t pp = pc + 16;                                                   \
        if (KC >= 3) {                                                           \
            uint32_t c2, c3, u0, u1;                                             \
            lds4(pp, c2, c3, u0, u1);                                            \
            Cs[2] = __uint_as_float(c2);                                         \
            Cs[3] = __uint_as_float(c3);                                         \
            pp += 16;                                                            \
        }                                                                        \
        const uint32_t tot = (counts & 7u) + ((counts >> 3) & 7u) +              \
                             ((counts >> 6) & 7u) + ((counts >> 9) & 7u);         \
        SPN_NEXT(pp + 16 * tot)                                                  \
        h_slp<SPN_SS(S), KC>(r, counts, bias, Cs, pp, e);                        \
    }
#define SPN_BODY_23(S) SPN_SLP_BODY(S, 2)
#define SPN_BODY_24(S) SPN_SLP_BODY(S, 3)
#define SPN_BODY_25(S) SPN_SLP_BODY(S, 4)
#define SPN_SLPU_BODY(S, KC)                                                     \
    {                                                                            \
        const float bias = __uint_as_float(cy);                                  \
        float Cs[4];                                                             \
        Cs[0] = __uint_as_float(cz);                                             \
        Cs[1] = __uint_as_float(cw);                                             \
        uint32_t ex, ey, ez, ew;                                                 \
        lds4(pc + 16, ex, ey, ez, ew);                                           \
        uint32_t fo[6];                                                          \
        if (KC == 2) {                                                           \
            fo[0] = ex & 0xffffu; fo[1] = ex >> 16;                              \
            fo[2] = ey & 0xffffu; fo[3] = ey >> 16;                              \
            fo[4] = 0; fo[5] = 0;                                                \
            Cs[2] = 0.f;                                                         \
        } else {                                                                 \
            Cs[2] = __uint_as_float(ex);                                         \
            fo[0] = ey & 0xffffu; fo[1] = ey >> 16;                              \
            fo[2] = ez & 0xffffu; fo[3] = ez >> 16;                              \
            fo[4] = ew & 0xffffu; fo[5] = ew >> 16;                              \
        }                                                                        \
        Cs[3] = 0.f;                                                             \
        const uint32_t pp = pc + 32;                                             \
        SPN_NEXT(pp + 16 * 2 * KC)                                               \
        h_slpu<SPN_SS(S), KC>(r, bias, Cs, fo, pp, e);                           \
    }
#define SPN_BODY_26(S) SPN_SLPU_BODY(S, 2)
#define SPN_BODY_27(S) SPN_SLPU_BODY(S, 3)
#define SPN_UNUSED_CASES case 476: case 477: case 478: case 479: case 480: case 481: case 482: case 483: case 484: case 485: case 486: case 487: case 488: case 489: case 490: case 491: case 492: case 493: case 494: case 495: case 496: case 497: case 498: case 499: case 500: case 501: case 502: case 503: case 504: case 505: case 506: case 507: case 508: case 509: case 510: case 511: return;

// Run one task's program (shared memory at byte address prog) for this
// thread's K samples.  All case labels 0..511 exist, so the dispatch is one
// unchecked jump-table lookup (build with nvcc -jtd 10).  Each case loads the
// next record right after reading its own operands (see SPN_NEXT).
template <int K, bool MARG, bool XS, int D>
__device__ __forceinline__ void run_task(uint32_t prog, const Env<K, MARG, XS> &e,
                                         ArgState<K> &am) {
    float r[D][K];
    uint32_t pc = prog;
    uint32_t cx, cy, cz, cw;
    lds4(pc, cx, cy, cz, cw);
    for (;;) {
        switch (cx & ((1u << CASE_BITS) - 1u)) {
            SPN_ALL_SP(SPN_CASE, 0)
            SPN_ALL_SP(SPN_CASE, 1)
            SPN_ALL_SP(SPN_CASE, 2)
            SPN_ALL_SP(SPN_CASE, 3)
            SPN_ALL_SP(SPN_CASE, 4)
            SPN_ALL_SP(SPN_CASE, 5)
            SPN_ALL_SP(SPN_CASE, 6)
            SPN_ALL_SP(SPN_CASE, 7)
            SPN_ALL_SP(SPN_CASE, 8)
            SPN_ALL_SP(SPN_CASE, 9)
            SPN_ALL_SP(SPN_CASE, 10)
            SPN_ALL_SP(SPN_CASE, 11)
            SPN_ALL_SP(SPN_CASE, 12)
            SPN_ALL_SP(SPN_CASE, 13)
            SPN_ALL_SP(SPN_CASE, 14)
            SPN_ALL_SP(SPN_CASE, 15)
            SPN_ALL_SP(SPN_CASE, 16)
            SPN_ALL_SP(SPN_CASE, 17)
            SPN_ALL_SP(SPN_CASE, 18)
            SPN_ALL_SP(SPN_CASE, 19)
            SPN_ALL_SP(SPN_CASE, 20)
            SPN_ALL_SP(SPN_CASE, 21)
            SPN_ALL_SP(SPN_CASE, 22)
            SPN_ALL_SP(SPN_CASE, 23)
            SPN_ALL_SP(SPN_CASE, 24)
            SPN_ALL_SP(SPN_CASE, 25)
            SPN_ALL_SP(SPN_CASE, 26)
            SPN_ALL_SP(SPN_CASE, 27)
            SPN_UNUSED_CASES
            default:
                __builtin_unreachable();
        }
    }
}

// Load this warp's tile of x (rows [base, base+nrows)) transposed into
// xw[f * tpw + s] (s = sample within the 32*K tile) with asynchronous 4-byte
// copies (cp.async, LDGSTS): all of them are in flight at once, then one wait.
// Rows past the end are zero-filled (src-size 0).
__device__ __forceinline__ void load_x_tile(float *xw, int tpw, const float *__restrict__ x,
                                            int64_t base, int nrows, int64_t ld, int F,
                                            int lane, int WT) {
    const int total = WT * F;
    int s = lane / F;
    int f = lane - s * F;
    const float *xb = x + base * ld;
    const uint32_t xa = smem_u32(xw);
    for (int idx = lane; idx < total; idx += 32) {
        const bool ok = s < nrows;
        const float *src = ok ? xb + (int64_t)s * ld + f : x;
        asm volatile("cp.async.ca.shared.global [%0], [%1], 4, %2;" ::"r"(
                         xa + 4u * (uint32_t)(f * tpw + s)),
                     "l"(src), "r"(ok ? 4 : 0)
                     : "memory");
        f += 32;
        while (f >= F) {
            f -= F;
            ++s;
        }
    }
    asm volatile("cp.async.commit_group;\ncp.async.wait_all;" ::: "memory");
}

template <int K, bool MARG, bool XS, int D>
__global__ void __launch_bounds__(K == 8 ? 256 : (K == 4 ? 384 : (K == 2 ? 768 : 512))) dag_eval_kernel(const KParams p) {
    extern __shared__ __align__(16) unsigned char smem_raw[];
    constexpr int WT = 32 * K;
    Rec *prog_s = reinterpret_cast<Rec *>(smem_raw);
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int nwarps = blockDim.x >> 5;
    const size_t xw_floats = XS ? (size_t)p.F * p.tpw : 0;
    const size_t warp_floats = xw_floats + (size_t)p.n_sslots * WT;
    float *warp_area = reinterpret_cast<float *>(smem_raw + (size_t)p.prog_cap * sizeof(Rec)) +
                       (size_t)warp * warp_floats;
    float *xw = warp_area;
    float *ss = warp_area + xw_floats;
    const int64_t gwarp = (int64_t)blockIdx.x * nwarps + warp;
    const int64_t total_warps = (int64_t)gridDim.x * nwarps;

    Env<K, MARG, XS> e;
    e.xs = pin_u32(smem_u32(xw + lane * K));
    e.ss = pin_u32(smem_u32(ss + lane * K));
    e.gs = reinterpret_cast<char *>(p.gslots + (size_t)gwarp * p.n_gslots * WT + lane * K);
    const uint32_t prog_a = pin_u32(smem_u32(prog_s));
    e.tables = p.tables;
    e.edges = p.edges;
    e.R = p.R;

    auto tile_begin = [&](int64_t base, ArgState<K> &am) {
        const int64_t rem = p.n - base;
        const int nrows = rem < WT ? (int)rem : WT;
        if constexpr (XS) {
            load_x_tile(xw, p.tpw, p.x, base, nrows, p.ld, p.F, lane, WT);
            __syncwarp();
        } else {
#pragma unroll
            for (int j = 0; j < K; ++j) {
                int64_t row = base + lane * K + j;
                row = row < p.n ? row : p.n - 1;
                e.xrow[j] = p.x + row * p.ld;
            }
        }
        const int64_t s0 = base + lane * K;
        const int64_t rv = p.n - s0;
        e.nvalid = rv <= 0 ? 0 : (rv < K ? (int)rv : K);
        e.out = p.out + (size_t)(rv > 0 ? s0 : 0) * p.R;
        am.init();
    };
    auto tile_end = [&](int64_t base, const ArgState<K> &am) {
        if (p.argmax) {
            const int64_t s0 = base + lane * K;
            FOR_K if (j < e.nvalid) p.argmax[s0 + j] = am.idx[j];
        }
        if constexpr (XS) __syncwarp();
    };

    if (p.n_tasks == 1) {
        const int len = p.first_task_len;
        for (int i = threadIdx.x; i < len + 2; i += blockDim.x)
            prog_s[i] = i < len ? p.prog[i] : make_end();
        __syncthreads();
        for (int64_t wt = gwarp; wt < p.n_wtiles; wt += total_warps) {
            const int64_t base = wt * WT;
            ArgState<K> am;
            tile_begin(base, am);
            run_task<K, MARG, XS, D>(prog_a, e, am);
            tile_end(base, am);
        }
    } else {
        const int64_t CT = (int64_t)nwarps * WT;
        const int64_t n_ctiles = (p.n + CT - 1) / CT;
        for (int64_t ct = blockIdx.x; ct < n_ctiles; ct += gridDim.x) {
            const int64_t base = ct * CT + (int64_t)warp * WT;
            const bool active = base < p.n;
            ArgState<K> am;
            if (active) tile_begin(base, am);
            for (int t = 0; t < p.n_tasks; ++t) {
                const int64_t b = p.task_off[t], len = p.task_off[t + 1] - b;
                __syncthreads();
                for (int64_t i = threadIdx.x; i < len + 2; i += blockDim.x)
                    prog_s[i] = i < len ? p.prog[b + i] : make_end();
                __syncthreads();
                if (active) run_task<K, MARG, XS, D>(prog_a, e, am);
            }
            if (active) tile_end(base, am);
        }
    }
}

// ---------------------------------------------------------------------------
// Host-side helpers, instantiated per K in dag_eval_k{1,2,4}.cu.
template <int K, bool MARG, bool XS, int D>
cudaError_t dag_eval_launch_t(const KParams &p, int grid, int block, size_t smem,
                              cudaStream_t st) {
    auto fn = dag_eval_kernel<K, MARG, XS, D>;
    // the attribute persists per function: set it only when a larger size is needed
    static size_t configured = 0;
    if (smem > configured) {
        cudaError_t err =
            cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        if (err != cudaSuccess) return err;
        configured = smem;
    }
    fn<<<grid, block, smem, st>>>(p);
    return cudaGetLastError();
}

template <int K, bool MARG, bool XS, int D>
int dag_eval_occupancy_t(int block, size_t smem) {
    auto fn = dag_eval_kernel<K, MARG, XS, D>;
    if (cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem) !=
        cudaSuccess)
        return 0;
    int nb = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, fn, block, smem) != cudaSuccess)
        return 0;
    return nb;
}

// maximum register-stack depth per samples-per-thread variant (registers:
// D x K stack values per thread)
template <int K>
constexpr int stack_depth() { return (K == 8 || K == 2) ? 10 : MAXD; }

#define SPNB_INSTANTIATE_K(K)                                                             \
    cudaError_t dag_eval_launch_k##K(const KParams &p, bool marg, bool xs, int grid,       \
                                     int block, size_t smem, cudaStream_t st) {            \
        constexpr int D = stack_depth<K>();                                               \
        if (marg) return xs ? dag_eval_launch_t<K, true, true, D>(p, grid, block, smem, st)  \
                            : dag_eval_launch_t<K, true, false, D>(p, grid, block, smem, st); \
        return xs ? dag_eval_launch_t<K, false, true, D>(p, grid, block, smem, st)           \
                  : dag_eval_launch_t<K, false, false, D>(p, grid, block, smem, st);         \
    }                                                                                     \
    int dag_eval_occupancy_k##K(bool marg, bool xs, int block, size_t smem) {             \
        constexpr int D = stack_depth<K>();                                               \
        if (marg) return xs ? dag_eval_occupancy_t<K, true, true, D>(block, smem)            \
                            : dag_eval_occupancy_t<K, true, false, D>(block, smem);          \
        return xs ? dag_eval_occupancy_t<K, false, true, D>(block, smem)                     \
                  : dag_eval_occupancy_t<K, false, false, D>(block, smem);                   \
    }

}  // namespace spnb
