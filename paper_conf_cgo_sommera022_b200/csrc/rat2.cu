// rat2.cu -- warp-specialised layered RAT-SPN kernel for sm_100a (KB2/KC2).
//
// Same method as rat_eval.cu (§V-B: leaf regions of
// factorised Gaussians, partitions = cross products of two regions, sum
// regions of S weighted sums; semantics of every node L82-86), restructured
// so that the FP32 leaf layer, the tensor-core contractions and the FP32
// epilogues of DIFFERENT regions run concurrently on one SM:
//
//   warps 0-7   two LEAF groups of 4 warps.  Group 0 evaluates the left
//               (A-side) leaf region of every bottom partition, group 1 the
//               right (B-side) one: L[i][m] = C_i - sum_v (a_iv x_mv - b_iv)^2
//               (log2), then the per-sample shift h = max_i L and the exps.
//               A side -> ea[i][m] (fp32, shared memory); B side -> the f16
//               UMMA operand image of eb'[m][j] = 2^(L_j - h + 15).
//   warps 8-11  EPILOGUE, one thread per sample (= TMEM lane).  For every
//               sum step: out_s = ha + hb + lg2(sum_i ea_i T[m,(s,i)]) - k_s,
//               T read from TMEM; upper-level shifts / exps / operand images;
//               the root's online log-sum-exp over repetitions.  Sum-region
//               outputs wait in TMEM "activation slots" for their parent.
//   warp 12     PRODUCER: TMA bulk copies of each leaf region's transposed
//               feature rows + parameter block, and of every weight group.
//   warp 13     MMA: tcgen05.mma (kind::f16, M=128) per weight group,
//               T[m,(s,i)] = sum_j eb'[m,j] W'[s,i,j] into a double-buffered
//               TMEM accumulator; completion by tcgen05.commit -> mbarrier.
//
// Every hand-off is an mbarrier ring (full/empty), so no role waits for the
// CTA: while the epilogue finishes repetition r's upper levels the leaf
// groups already compute the next leaf regions and the producer streams
// the next weight groups.  One persistent CTA per SM walks 128-sample tiles.
#include <cuda_fp16.h>
#include <cuda_runtime.h>
#include <math_constants.h>
#include <stdint.h>

#include <algorithm>

#include "layered.h"

namespace spnb {
namespace r2 {

constexpr int RT = 128;           // samples per tile = UMMA M = TMEM lanes
// 16 warps = 4 warpgroups: leaf, epilogue (accumulator A), epilogue
// (accumulator B), {leaf producer, MMA, weight producer, idle}.  setmaxnreg
// moves registers from the last warpgroup (56 each) to the other three
// (152 each): 3*152 + 56 = 512 per SMSP lane.
#ifndef R2_WARPS
#define R2_WARPS 16
#endif
#if R2_WARPS == 20
// 20 warps: two leaf groups (left / right regions), 8 epilogue warps, producers
// setmaxnreg moves registers only within the CTA's launch allocation
// (640 threads x 96): 8*96 + 8*120 + 4*40 = 1888 <= 20*96 per lane
constexpr int NLG = 2, EPI_COLS = 40;
constexpr int REG_LEAF = 96, REG_EPI = 120, REG_PROD = 40;
#else
// launch allocation 512 threads x 128: 4*152 + 8*152 + 4*56 = 2048 = 16*128 per lane
constexpr int NLG = 1, EPI_COLS = 80;
constexpr int REG_LEAF = 152, REG_EPI = 152, REG_PROD = 56;
#endif
#ifndef R2_NAB
#define R2_NAB 3  // left / right leaf-output slots (the leaf warps' run-ahead)
#endif
constexpr int NAB = R2_NAB;
#ifndef EPI_SHARE
#define EPI_SHARE 0  // 1: both epilogue warps of a lane quarter drain every group (measured slower)
#endif
#ifndef R2_XROWS_CPASYNC
#define R2_XROWS_CPASYNC 0  // 1: leaf feature rows by cp.async (LSU) instead of per-row bulk copies (TMA)
#endif
#ifndef R2_MMA_PERGROUP
// 1: the MMA warp issues each group as soon as its own accumulator is
// drained (C5 +5% over waiting for both accumulators of a pair)
#define R2_MMA_PERGROUP 1
#endif
#ifndef R2_EPI_RELEASE
// 1: the epilogue, having observed a group's T_FULL, releases its weight slot
// (and after the step's last group the step's operand image) with a plain
// mbarrier arrive, so the MMA warp issues one tcgen05.commit per group
// instead of two (+ one per step); needs R2_MMA_PERGROUP.  Measured 2%
// slower on C5 (the release moves onto the epilogue's critical path)
#define R2_EPI_RELEASE 0
#endif
static_assert(!(EPI_SHARE && R2_EPI_RELEASE), "R2_EPI_RELEASE needs one drainer per group");
#ifndef R2_MMA_INTERLEAVE
#define R2_MMA_INTERLEAVE 0  // 1: K-steps of the two accumulators interleaved (round-1 order; measured slower)
#endif
#ifndef R2_UPIMG_H
#define R2_UPIMG_H 0  // epilogue warp (0: accumulator A side, 1: B side) that writes the UP operand image
#endif
#ifndef LEAF_SPT
// samples per leaf thread: 8 = one region per 2 warps, the two leaf pairs on
// alternate (left / right) regions (C5 +4%, C4 +5% over 4 = one region per
// 4 warps once the MMA issues per group; scripts/gpu/r02/r02_leaf.sh)
#define LEAF_SPT 8
#endif
constexpr int NTHREADS = (4 * NLG + 12) * 32;
// registers per thread of the launch (65536 / NTHREADS rounded down to 8):
// the pool setmaxnreg redistributes; rat2_launch refuses a build whose
// register count differs (an unbalanced budget would block setmaxnreg.inc)
constexpr int LAUNCH_REGS = (65536 / NTHREADS) / 8 * 8;
static_assert(4 * NLG * REG_LEAF + 8 * REG_EPI + 4 * REG_PROD <= (4 * NLG + 12) * LAUNCH_REGS,
              "setmaxnreg budget exceeds the launch allocation");
constexpr int W_EPI0 = 4 * NLG;   // epilogue warps: two per TMEM lane quarter
constexpr int W_PROD = W_EPI0 + 8, W_MMA = W_PROD + 1, W_WPROD = W_PROD + 2;
constexpr float EB_SHIFT = 15.f;  // eb' = 2^(b - hb + 15): f16-normal down to eb = 2^-29
// TMEM accumulators: A = columns [0, CA), B = [CA, CA + CB); the groups of a
// step alternate A, B (layered.h R2Step).  FMA leaves: 240 + 160; tensor-core
// leaves (LTC): 160 + 160, then the leaf accumulator (48 columns); the
// activation slots and root columns follow.  LTC keeps two left/right
// leaf-output slots (its feature image takes the third one's shared memory).
template <bool LTC>
struct Cols {
    static constexpr int A = LTC ? R2T_COLS_A : R2_COLS_A;
    static constexpr int B = LTC ? R2T_COLS_B : R2_COLS_B;
    static constexpr int L = A + B;
    static constexpr int SLOTS = A + B + (LTC ? R2T_COLS_L : 0);
    static constexpr int NAB = LTC ? 2 : R2_NAB;
};

__device__ __forceinline__ float ex2(float x) {
    float y;
    asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
    return y;
}
__device__ __forceinline__ float lg2(float x) {
    float y;
    asm("lg2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
    return y;
}
__device__ __forceinline__ float maxnan(float a, float b) {
    float r;
    asm("max.NaN.f32 %0, %1, %2;" : "=f"(r) : "f"(a), "f"(b));
    return r;
}
// log2(2^a + 2^b), NaN-propagating, -inf safe
__device__ __forceinline__ float lse2(float a, float b) {
    const float hi = maxnan(a, b), lo = fminf(a, b);
    return hi + lg2(1.f + ex2(lo - fmaxf(hi, -1e30f)));
}
__device__ __forceinline__ uint32_t smem_u32(const void *p) {
    return (uint32_t)__cvta_generic_to_shared(p);
}

// ---- mbarriers -------------------------------------------------------------
__device__ __forceinline__ void bar_init(uint32_t b, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(b), "r"(count));
}
// plain try_wait (the instruction itself suspends the warp for a
// hardware-defined time).  Measured alternatives (C5, scripts/gpu/r02_*.sh):
// a 10 ms suspend-time hint (R2_WAIT_HINT; compiles to a NANOSLEEP.SYNCS
// loop) -1%, test_wait + nanosleep 32 / 128 ns (R2_WAIT_SLEEP) -4% / -1%.
// R2_WATCHDOG builds (development): a wait that has not completed after
// 2^34 cycles (~9 s; a 128-sample tile takes ~6 ms on C5) is a protocol
// deadlock -- trap so the launch fails instead of hanging the device.  Off
// in the product build (the clock reads cost ~7% on C5).
__device__ __forceinline__ void bar_wait(uint32_t b, uint32_t parity) {
    uint32_t done = 0;
#ifdef R2_WATCHDOG
    long long t0 = 0;
#endif
    while (true) {
#if defined(R2_WAIT_SLEEP)
        // poll without parking on the barrier unit: test, then sleep
        asm volatile(
            "{\n\t.reg .pred p;\n\tmbarrier.test_wait.parity.shared::cta.b64 p, [%1], %2;\n\t"
            "selp.u32 %0, 1, 0, p;\n\t}\n"
            : "=r"(done)
            : "r"(b), "r"(parity)
            : "memory");
        if (done) break;
        __nanosleep(R2_WAIT_SLEEP);
        continue;
#endif
#ifndef R2_WAIT_HINT
        asm volatile(
            "{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\t"
            "selp.u32 %0, 1, 0, p;\n\t}\n"
            : "=r"(done)
            : "r"(b), "r"(parity)
            : "memory");
#else
        asm volatile(
            "{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2, %3;\n\t"
            "selp.u32 %0, 1, 0, p;\n\t}\n"
            : "=r"(done)
            : "r"(b), "r"(parity), "r"(0x989680u)
            : "memory");
#endif
        if (done) break;
#ifdef R2_WATCHDOG
        long long t;
        asm volatile("mov.u64 %0, %%clock64;" : "=l"(t));
        if (t0 == 0) t0 = t;
        else if (t - t0 > (1ll << 34)) __trap();
#endif
    }
}
__device__ __forceinline__ void bar_arrive(uint32_t b) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(b) : "memory");
}
__device__ __forceinline__ void bar_expect_tx(uint32_t b, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(b), "r"(bytes)
                 : "memory");
}
__device__ __forceinline__ void bulk_g2s(uint32_t dst, const void *src, uint32_t bytes,
                                         uint32_t b) {
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
            dst),
        "l"(src), "r"(bytes), "r"(b)
        : "memory");
}
__device__ __forceinline__ void fence_async_smem() {
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}

// ---- tcgen05 -----------------------------------------------------------------
__device__ __forceinline__ uint64_t umma_desc(uint32_t addr, uint32_t lbo, uint32_t sbo) {
    // K-major, no swizzle: core matrices of 8 rows x 16 bytes; LBO = stride
    // between core matrices along K, SBO = along M/N; version 1 (sm_100)
    uint64_t d = 0;
    d |= (uint64_t)((addr >> 4) & 0x3FFFu);
    d |= (uint64_t)((lbo >> 4) & 0x3FFFu) << 16;
    d |= (uint64_t)((sbo >> 4) & 0x3FFFu) << 32;
    d |= (uint64_t)1 << 46;
    return d;
}
__device__ __forceinline__ void umma_f16(uint32_t d_tmem, uint64_t a, uint64_t b, uint32_t idesc,
                                         uint32_t acc) {
    asm volatile(
        "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}\n" ::"r"(d_tmem),
        "l"(a), "l"(b), "r"(idesc), "r"(acc));
}
__device__ __forceinline__ void umma_commit(uint32_t b) {
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(b)
                 : "memory");
}
__device__ __forceinline__ void tc_fence_before() {
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
}
__device__ __forceinline__ void tc_fence_after() {
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
}
__device__ __forceinline__ void tmem_ld8(uint32_t taddr, float *v) {
    uint32_t r[8];
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x8.b32 {%0, %1, %2, %3, %4, %5, %6, %7}, [%8];"
        : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]),
          "=r"(r[7])
        : "r"(taddr));
#pragma unroll
    for (int k = 0; k < 8; ++k) v[k] = __uint_as_float(r[k]);
}
__device__ __forceinline__ void tmem_ld16(uint32_t taddr, float *v) {
    uint32_t r[16];
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0, %1, %2, %3, %4, %5, %6, %7, %8, %9, %10, %11, "
        "%12, %13, %14, %15}, [%16];"
        : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]),
          "=r"(r[7]), "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]),
          "=r"(r[14]), "=r"(r[15])
        : "r"(taddr));
#pragma unroll
    for (int k = 0; k < 16; ++k) v[k] = __uint_as_float(r[k]);
}
__device__ __forceinline__ void tmem_ld4(uint32_t taddr, float *v) {
    uint32_t r[4];
    asm volatile("tcgen05.ld.sync.aligned.32x32b.x4.b32 {%0, %1, %2, %3}, [%4];"
                 : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3])
                 : "r"(taddr));
#pragma unroll
    for (int k = 0; k < 4; ++k) v[k] = __uint_as_float(r[k]);
}
__device__ __forceinline__ void tmem_ld1(uint32_t taddr, float &v) {
    uint32_t r;
    asm volatile("tcgen05.ld.sync.aligned.32x32b.x1.b32 {%0}, [%1];" : "=r"(r) : "r"(taddr));
    v = __uint_as_float(r);
}
__device__ __forceinline__ void tmem_st1(uint32_t taddr, float v) {
    asm volatile("tcgen05.st.sync.aligned.32x32b.x1.b32 [%0], {%1};" ::"r"(taddr),
                 "r"(__float_as_uint(v)));
}
__device__ __forceinline__ void tmem_wait_ld() {
    asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
}
__device__ __forceinline__ void tmem_wait_st() {
    asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
}

// byte offset of element (row, k) of a K-major no-swizzle f16 operand image
// with RT rows
__device__ __forceinline__ uint32_t img_off(int row, int k) {
    return (uint32_t)((k >> 3) * (RT * 16) + (row >> 3) * 128 + (row & 7) * 16 + (k & 7) * 2);
}
// two floats -> packed f16x2 with one cvt.rn.f16x2.f32 (a in the low half)
__device__ __forceinline__ uint32_t pack_h2(float a, float b) {
    uint32_t r;
    asm("cvt.rn.f16x2.f32 %0, %1, %2;" : "=r"(r) : "f"(b), "f"(a));
    return r;
}
// hi/lo split of a pair: hi = f16(v), lo = f16(v - hi)
__device__ __forceinline__ void split_h2(float a, float b, uint32_t &hi, uint32_t &lo) {
    const __half ha = __float2half_rn(a), hb = __float2half_rn(b);
    hi = (uint32_t)__half_as_ushort(ha) | ((uint32_t)__half_as_ushort(hb) << 16);
    lo = pack_h2(a - __half2float(ha), b - __half2float(hb));
}

// optional phase-cycle counters (R2Params::prof, SPNB_PROFILE=1): every role
// attributes the cycles since its previous mark to a phase; lane 0 of each
// role's warps adds them to prof[role * 8 + phase] at exit
__device__ __forceinline__ long long clk64() {
    long long t;
    asm volatile("mov.u64 %0, %%clock64;" : "=l"(t));
    return t;
}
#ifdef R2_TRACE
// development timeline (R2_TRACE builds with SPNB_PROFILE=1): CTA 0's phase
// marks as (clock, warp << 8 | phase) pairs in per-warp regions (plain
// stores, no atomics on the timed path), read back by spnb_r2_trace
constexpr unsigned TRACE_W = 8192;  // events per warp
constexpr unsigned TRACE_N = 16 * TRACE_W;
__device__ unsigned long long g_trace[2 * TRACE_N];
#endif
struct Prof {
    unsigned long long *acc;  // shared-memory counters of this role (nullptr: off)
    long long t;
#ifdef R2_TRACE
    unsigned cnt = 0;
#endif
    __device__ Prof(unsigned long long *a, bool on) : acc(on ? a : nullptr), t(clk64()) {}
    __device__ __forceinline__ void mark(int k) {
        if (acc) {
            const long long now = clk64();
#ifdef R2_TRACE
            if ((threadIdx.x & 31) == 0 && blockIdx.x == 0 && cnt < TRACE_W) {
                const unsigned i = (threadIdx.x >> 5) * TRACE_W + cnt++;
                g_trace[2 * i] = (unsigned long long)now;
                g_trace[2 * i + 1] = ((threadIdx.x >> 5) << 8) | (unsigned)k;
            }
#else
            if ((threadIdx.x & 31) == 0) atomicAdd(acc + k, (unsigned long long)(now - t));
#endif
            t = now;
        }
    }
};

// shared-memory layout: barrier indices
enum {
    B_IN_FULL = 0,    // [4]
    B_IN_EMPTY = 4,   // [4]
    B_A_FULL = 8,     // [4] (NAB used)
    B_A_EMPTY = 12,   // [4]
    B_B_FULL = 16,    // [4]
    B_B_EMPTY = 20,   // [4]
    B_U_FULL = 24,
    B_U_EMPTY = 25,
    B_W_FULL = 26,    // [8]
    B_W_EMPTY = 34,   // [8]
    B_T_FULL = 42,    // [2]
    B_T_EMPTY = 44,   // [2]
    B_F_FULL = 46,    // tensor-core leaves: feature image written (leaf warps -> leaf MMA)
    B_LT_FULL = 47,   // tensor-core leaves: leaf accumulator ready (leaf MMA commit -> leaf warps)
    B_COUNT = 48
};

struct Smem {
    // offsets are read from the kernel parameter (constant bank) at each use
    // instead of being copied into registers that live across the role loops
    uint8_t *base;
    const R2Params &p;
    __device__ Smem(uint8_t *b, const R2Params &pp) : base(b), p(pp) {}
    __device__ uint32_t bar(int i) const { return smem_u32(base + p.off_bar) + 8u * (uint32_t)i; }
    // profiling counters: [4 roles][8] after the barriers and the TMEM slot
    __device__ unsigned long long *prof(int role) const {
        return reinterpret_cast<unsigned long long *>(base + p.off_bar + 8 * B_COUNT + 16) + role * 8;
    }
    __device__ float *in_x(int s) const {
        return reinterpret_cast<float *>(base + p.off_in + s * p.in_bytes);
    }
    __device__ float *in_prm(int s) const { return in_x(s) + p.max_vars * RT; }
    __device__ float *ea(int s) const {
        return reinterpret_cast<float *>(base + p.off_ea + s * p.ea_bytes);
    }
    // per A-slot: ea[I][RT], ha[RT], hb[RT]
    __device__ float *ha(int s) const { return ea(s) + p.I * RT; }
    __device__ float *hb(int s) const { return ha(s) + RT; }
    __device__ uint8_t *bimg(int s) const { return base + p.off_bimg + s * p.bimg_bytes; }
    __device__ uint8_t *uimg() const { return base + p.off_uimg; }
    __device__ uint8_t *wbuf(int s) const { return base + p.off_w + s * p.w_bytes; }
    // tensor-core leaves: feature image (hi part, lo part after it) and the
    // parameter image inside input slot s
    __device__ uint8_t *fimg() const { return base + p.off_f; }
    __device__ uint8_t *in_pimg(int s) const {
        return reinterpret_cast<uint8_t *>(in_x(s)) + p.pimg_off;
    }
};

// ============================================================== LEAF groups
// Thread (gw, q, b): samples m0 = 32 gw + 4 q .. +3, distributions
// d0 = b DPB .. +DPB-1 (DPB = I / 4).  Per variable: one LDS.128 of the four
// samples' features (a warp reads 128 contiguous bytes) and DPB/2 LDS.128 of
// (a, b) pairs (4 distinct addresses per warp), then 2 DPB FFMA2.
template <int DPB, int SPT, bool MARG>
__device__ __forceinline__ void leaf_compute(const float *xs, const float *prm, int V, int I,
                                             int m0, int d0, float (&acc)[DPB][SPT]) {
    const float *C = prm + 2 * V * I;
#pragma unroll
    for (int d = 0; d < DPB; ++d) {
        const float c = C[d0 + d];
#pragma unroll
        for (int k = 0; k < SPT; ++k) acc[d][k] = c;
    }
    const float K0 = -1.0901312512f;  // 0.5 * log2(ln2 / pi): c_v = log2(a) + K0
    const float4 *ab4 = reinterpret_cast<const float4 *>(prm + 2 * d0);
    const int vstride = I / 2;  // float4 per variable
#pragma unroll 2
    for (int v = 0; v < V; ++v) {
        float xv[SPT];
#pragma unroll
        for (int c = 0; c < SPT; c += 4) {
            const float4 x4 = *reinterpret_cast<const float4 *>(xs + v * RT + m0 + c);
            xv[c] = x4.x; xv[c + 1] = x4.y; xv[c + 2] = x4.z; xv[c + 3] = x4.w;
        }
        float2 q[DPB];
#pragma unroll
        for (int k = 0; k < DPB / 2; ++k) {
            const float4 t = ab4[v * vstride + k];
            q[2 * k] = make_float2(t.x, t.y);
            q[2 * k + 1] = make_float2(t.z, t.w);
        }
        bool anynan = false;
        if constexpr (MARG) {
#pragma unroll
            for (int k = 0; k < SPT; ++k) anynan |= xv[k] != xv[k];
        }
        if (MARG && anynan) {
#pragma unroll
            for (int d = 0; d < DPB; ++d) {
                const float cc = lg2(q[d].x) + K0;
#pragma unroll
                for (int k = 0; k < SPT; ++k) {
                    const bool nan = xv[k] != xv[k];
                    const float t = fmaf(q[d].x, xv[k], -q[d].y);
                    acc[d][k] = fmaf(-(nan ? cc : t), nan ? 1.f : t, acc[d][k]);
                }
            }
        } else {
#pragma unroll
            for (int d = 0; d < DPB; ++d) {
                const float2 a2 = make_float2(q[d].x, q[d].x), nb2 = make_float2(-q[d].y, -q[d].y);
#pragma unroll
                for (int k = 0; k < SPT; k += 2) {
                    const float2 t = __ffma2_rn(make_float2(xv[k], xv[k + 1]), a2, nb2);
                    const float2 r = __ffma2_rn(make_float2(-t.x, -t.y), t,
                                                make_float2(acc[d][k], acc[d][k + 1]));
                    acc[d][k] = r.x;
                    acc[d][k + 1] = r.y;
                }
            }
        }
    }
}

// leaf warps: LW = 4 NLG; a group of WPG = 16 / LEAF_SPT warps evaluates one
// leaf region for the tile's 128 samples (thread = LEAF_SPT samples x I/4
// distributions: lane = 8 sample groups x 4 distribution blocks); the LW /
// WPG groups take consecutive regions (left A / right B alternate)
constexpr int WPG = 16 / LEAF_SPT;
constexpr int NGRP = 4 * NLG / WPG;

template <int DPB, bool MARG>
__device__ void leaf_role(const R2Params &p, const Smem &sm, const int32_t *leaf_steps,
                          int n_leaf, int warp, int lane) {
    constexpr int SPT = LEAF_SPT;
    const int g = warp / WPG, gw = warp % WPG;
    const int q = lane >> 2, b = lane & 3;
    const int m0 = gw * (RT / WPG) + q * SPT, d0 = b * DPB;
    const int I = p.I;
    const int64_t n_tiles = (p.n + RT - 1) / RT;
    uint32_t li = (uint32_t)g;  // global leaf-region counter (step NGRP); even: A side, odd: B side
    Prof pf(sm.prof(0), p.prof != nullptr);  // 0 wait input, 1 compute, 2 shifts, 3 wait output slot, 4 exps + write
    for (int64_t tile = blockIdx.x; tile < n_tiles; tile += gridDim.x) {
        for (int l = g; l < n_leaf; l += NGRP, li += NGRP) {
            const bool side_b = (l & 1) != 0;  // leaf regions alternate left (A) / right (B)
            const uint32_t j = li >> 1;         // bottom partition
            const R2Step &st = p.steps[leaf_steps[l]];
            const int s = (int)(li % (uint32_t)p.n_in);
            bar_wait(sm.bar(B_IN_FULL + s), (li / (uint32_t)p.n_in) & 1u);
            pf.mark(0);
            float acc[DPB][SPT];
#ifdef R2_KO_LEAF  // knockout (critical-path experiments; wrong results): no leaf FMAs
            leaf_compute<DPB, SPT, MARG>(sm.in_x(s), sm.in_prm(s), 0, I, m0, d0, acc);
#else
            leaf_compute<DPB, SPT, MARG>(sm.in_x(s), sm.in_prm(s), st.n_vars, I, m0, d0, acc);
#endif
            // the slot's next fill is an async-proxy (TMA) write: order this
            // warp's generic-proxy reads before the release of the slot
            fence_async_smem();
            __syncwarp();
            if (lane == 0) bar_arrive(sm.bar(B_IN_EMPTY + s));
            pf.mark(1);
            // per-sample shift over the I distributions: local max over DPB,
            // then across the 4 lanes of the sample group (xor 1, 2)
            float h[SPT];
#pragma unroll
            for (int k = 0; k < SPT; ++k) {
                float v = acc[0][k];
#pragma unroll
                for (int d = 1; d < DPB; ++d) v = maxnan(v, acc[d][k]);
                v = maxnan(v, __shfl_xor_sync(0xffffffffu, v, 1));
                v = maxnan(v, __shfl_xor_sync(0xffffffffu, v, 2));
                h[k] = v;
            }
            const int ab = (int)(j % NAB);
            const uint32_t ph = (j / NAB) & 1u;
            pf.mark(2);
            // both sides wait for the A slot (it also carries hb)
            bar_wait(sm.bar(B_A_EMPTY + ab), ph ^ 1u);
            if (side_b) bar_wait(sm.bar(B_B_EMPTY + ab), ph ^ 1u);
            pf.mark(3);
            if (!side_b) {
                float *ea = sm.ea(ab);
#pragma unroll
                for (int d = 0; d < DPB; ++d) {
#pragma unroll
                    for (int c = 0; c < SPT; c += 4) {
                        float e[4];
#pragma unroll
                        for (int k = 0; k < 4; ++k) e[k] = ex2(acc[d][c + k] - fmaxf(h[c + k], -1e30f));
                        *reinterpret_cast<float4 *>(ea + (d0 + d) * RT + m0 + c) =
                            make_float4(e[0], e[1], e[2], e[3]);
                    }
                }
                if (b == 0)
#pragma unroll
                    for (int c = 0; c < SPT; c += 4)
                        *reinterpret_cast<float4 *>(sm.ha(ab) + m0 + c) =
                            make_float4(h[c], h[c + 1], h[c + 2], h[c + 3]);
                bar_arrive(sm.bar(B_A_FULL + ab));
            } else {
                uint8_t *img = sm.bimg(ab);
                const int part = p.bimg_bytes / 2;  // lo image after hi (prec 3)
#pragma unroll
                for (int k = 0; k < SPT; ++k) {
                    const float hc = fmaxf(h[k], -1e30f) - EB_SHIFT;
#pragma unroll
                    for (int d = 0; d < DPB; d += 2) {
                        const float e0 = ex2(acc[d][k] - hc), e1 = ex2(acc[d + 1][k] - hc);
                        const uint32_t o = img_off(m0 + k, d0 + d);
                        if (p.prec == 3) {
                            uint32_t hi, lo;
                            split_h2(e0, e1, hi, lo);
                            *reinterpret_cast<uint32_t *>(img + o) = hi;
                            *reinterpret_cast<uint32_t *>(img + part + o) = lo;
                        } else {
                            *reinterpret_cast<uint32_t *>(img + o) = pack_h2(e0, e1);
                        }
                    }
                }
                if (b == 0)
#pragma unroll
                    for (int c = 0; c < SPT; c += 4)
                        *reinterpret_cast<float4 *>(sm.hb(ab) + m0 + c) =
                            make_float4(h[c] - EB_SHIFT, h[c + 1] - EB_SHIFT, h[c + 2] - EB_SHIFT,
                                        h[c + 3] - EB_SHIFT);
                fence_async_smem();
                bar_arrive(sm.bar(B_B_FULL + ab));
            }
            pf.mark(4);
        }
    }
}

// ============================================================== PRODUCERS
// Two warps so leaf inputs never queue behind weight groups (the weight
// ring drains at the pace of the epilogue): warp W_PROD streams each leaf
// region's feature rows + parameter block, warp W_WPROD every weight group.
template <bool LTC, bool MARG>
__device__ void leaf_producer_role(const R2Params &p, const Smem &sm, const int32_t *leaf_steps,
                                   int n_leaf, int lane) {
    const int64_t n_tiles = (p.n + RT - 1) / RT;
    uint32_t li = 0;
    Prof pf(sm.prof(3), p.prof != nullptr);  // 0 wait leaf slot, 7 issue
    for (int64_t tile = blockIdx.x; tile < n_tiles; tile += gridDim.x) {
        const int64_t base = tile * RT;
        for (int l = 0; l < n_leaf; ++l, ++li) {
            const R2Step &st = p.steps[leaf_steps[l]];
            const int s = (int)(li % (uint32_t)p.n_in);
            pf.mark(7);
            bar_wait(sm.bar(B_IN_EMPTY + s), ((li / (uint32_t)p.n_in) & 1u) ^ 1u);
            pf.mark(0);
            const uint32_t full = sm.bar(B_IN_FULL + s);
            const uint32_t pbytes = (uint32_t)st.blk_floats * 4;
            const uint32_t dst = smem_u32(sm.in_x(s));
#if R2_XROWS_CPASYNC
            // feature rows through the LSU path (cp.async, 16 B per lane per
            // row): hundreds of 512-byte bulk copies per tile would queue
            // ahead of the weight groups in the TMA unit.  Each lane's
            // cp.async.mbarrier.arrive adds a pending arrival now and
            // completes it when its copies land, so the slot's phase waits
            // for them; issued before lane 0's expect_tx arrive.
            if (!LTC) {
                for (int v0 = 0; v0 < st.n_vars; v0 += 32) {
                    const int vl = v0 + lane < st.n_vars ? __ldg(p.vars + st.vars_off + v0 + lane) : 0;
                    const int nv = min(32, st.n_vars - v0);
                    for (int v = 0; v < nv; ++v) {
                        const int f = __shfl_sync(0xffffffffu, vl, v);
                        const float *src = p.xT + (int64_t)f * p.ldT + base + lane * 4;
                        asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(
                                         dst + (uint32_t)((v0 + v) * RT * 4 + lane * 16)),
                                     "l"(src)
                                     : "memory");
                    }
                }
                asm volatile("cp.async.mbarrier.arrive.shared::cta.b64 [%0];" ::"r"(full) : "memory");
                __syncwarp();
                if (lane == 0) {
                    bar_expect_tx(full, pbytes);
                    bulk_g2s(smem_u32(sm.in_prm(s)), p.fparams + st.blk_off, pbytes, full);
                }
                __syncwarp();
                continue;
            }
#endif
            if (lane == 0) {
                if constexpr (LTC) {
                    // centres + the query's parameter image (hi, lo)
                    const uint32_t ib = 2u * (uint32_t)(MARG ? st.wbytes_b : st.wbytes_a);
                    bar_expect_tx(full, (uint32_t)st.n_vars * RT * 4 + pbytes + ib);
                    bulk_g2s(smem_u32(sm.in_prm(s)), p.fparams + st.blk_off, pbytes, full);
                    bulk_g2s(smem_u32(sm.in_pimg(s)), p.wimg + st.w_off + (MARG ? 2 * st.wbytes_a : 0), ib,
                             full);
                } else {
                    bar_expect_tx(full, (uint32_t)st.n_vars * RT * 4 + pbytes);
                    bulk_g2s(smem_u32(sm.in_prm(s)), p.fparams + st.blk_off, pbytes, full);
                }
            }
            __syncwarp();
            for (int v = lane; v < st.n_vars; v += 32) {
                const int f = __ldg(p.vars + st.vars_off + v);
                bulk_g2s(dst + v * RT * 4, p.xT + (int64_t)f * p.ldT + base, RT * 4, full);
            }
        }
    }
    pf.mark(7);
}

// the fields of a sum step the MMA / epilogue / weight roles use, loaded once
// per step into registers (held by reference, every use in a loop would be a
// dependent global load on the role's critical path)
struct SumStep {
    int type, root, n_out, na, kpad, n_groups, spg_a, ncol_a, spg_b, ncol_b, slot_a, slot_b,
        slot_out;
    int64_t blk_off, w_off, wbytes_a, wbytes_b;
};
__device__ __forceinline__ SumStep load_sum_step(const R2Step *steps, const int32_t *idx, int si) {
    const R2Step *q = steps + __ldg(idx + si);
    SumStep r;
    r.type = __ldg(&q->type);
    r.root = __ldg(&q->root);
    r.n_out = __ldg(&q->n_out);
    r.na = __ldg(&q->na);
    r.kpad = __ldg(&q->kpad);
    r.n_groups = __ldg(&q->n_groups);
    r.spg_a = __ldg(&q->spg_a);
    r.ncol_a = __ldg(&q->ncol_a);
    r.spg_b = __ldg(&q->spg_b);
    r.ncol_b = __ldg(&q->ncol_b);
    r.slot_a = __ldg(&q->slot_a);
    r.slot_b = __ldg(&q->slot_b);
    r.slot_out = __ldg(&q->slot_out);
    r.blk_off = __ldg(&q->blk_off);
    r.w_off = __ldg(&q->w_off);
    r.wbytes_a = __ldg(&q->wbytes_a);
    r.wbytes_b = __ldg(&q->wbytes_b);
    return r;
}

// group gi of a sum step: first sum, number of sums (0: empty), MMA columns,
// image byte offset relative to w_off and bytes of one part image
struct GroupInfo {
    int s0, ns, ncol;
    int64_t off, bytes;
};
__device__ __forceinline__ GroupInfo group_info(const SumStep &st, int gi) {
    const bool b = gi & 1;
    const int pair = gi >> 1;
    GroupInfo g;
    g.s0 = pair * (st.spg_a + st.spg_b) + (b ? st.spg_a : 0);
    g.ns = max(0, min(b ? st.spg_b : st.spg_a, st.n_out - g.s0));
    g.ncol = b ? st.ncol_b : st.ncol_a;
    g.bytes = b ? st.wbytes_b : st.wbytes_a;
    g.off = (int64_t)pair * 2 * (st.wbytes_a + st.wbytes_b) + (b ? 2 * st.wbytes_a : 0);
    return g;
}

__device__ void weight_producer_role(const R2Params &p, const Smem &sm, const int32_t *sum_steps,
                                     int n_sum, int lane) {
    const int64_t n_tiles = (p.n + RT - 1) / RT;
    uint32_t w_idx = 0, w_ph = 0;
    const uint32_t n_w = (uint32_t)p.n_w;
    const int parts = p.prec == 3 ? 2 : 1;
    Prof pf(sm.prof(3), p.prof != nullptr);  // 2 wait weight slot, 7 issue
    for (int64_t tile = blockIdx.x; tile < n_tiles; tile += gridDim.x) {
        for (int si = 0; si < n_sum; ++si) {
            const SumStep st = load_sum_step(p.steps, sum_steps, si);
            for (int gi = 0; gi < st.n_groups; ++gi) {
                const GroupInfo gr = group_info(st, gi);
                if (gr.ns == 0) continue;  // empty group: no weights (the MMA skips it too)
                pf.mark(7);
                bar_wait(sm.bar(B_W_EMPTY) + 8u * w_idx, w_ph ^ 1u);
                pf.mark(2);
                const uint32_t full = sm.bar(B_W_FULL) + 8u * w_idx;
                if (lane == 0) {
                    const uint32_t gb = (uint32_t)gr.bytes;
#ifdef R2_KO_W  // knockout (wrong results): weight slots handed over without copies
                    bar_arrive(full);
#else
                    bar_expect_tx(full, gb * parts);
                    const uint8_t *src = p.wimg + st.w_off + gr.off;
                    for (int pt = 0; pt < parts; ++pt)
                        bulk_g2s(smem_u32(sm.wbuf((int)w_idx)) + pt * (uint32_t)p.max_wgroup,
                                 src + (size_t)pt * gb, gb, full);
#endif
                }
                __syncwarp();
                if (++w_idx == n_w) {
                    w_idx = 0;
                    w_ph ^= 1u;
                }
            }
        }
    }
    pf.mark(7);
}

// ============================================================== MMA issuer
// Per pair of groups (A, B) the K-steps of the two accumulators are
// interleaved (consecutive MMAs into one accumulator serialise on its
// latency, ~170 cycles per step on B200 whatever N; two chains overlap).
// Ring positions advance incrementally (no runtime division); descriptors
// are built once per group and advanced along K by adding byte offset >> 4
// to the start-address field (shared addresses < 256 KB never carry).
__device__ __forceinline__ uint64_t desc_hi(uint32_t lbo, uint32_t sbo) {
    return ((uint64_t)((lbo >> 4) & 0x3FFFu) << 16) | ((uint64_t)((sbo >> 4) & 0x3FFFu) << 32) |
           ((uint64_t)1 << 46);
}
template <bool LTC>
__device__ void mma_role(const R2Params &p, const Smem &sm, const int32_t *sum_steps, int n_sum,
                         uint32_t tmem, int lane) {
    const int64_t n_tiles = (p.n + RT - 1) / RT;
    uint32_t kb = 0, ku = 0, tp = 0;  // BOT / UP operand counters, accumulator-pair counter
    uint32_t w_idx = 0, w_ph = 0;     // next weight-ring slot and its phase
    const uint32_t n_w = (uint32_t)p.n_w;
    const uint32_t lbo_a = RT * 16;
    const uint64_t a_hi_bits = desc_hi(lbo_a, 128);
    const uint32_t wbase = smem_u32(sm.wbuf(0)), wstride = (uint32_t)p.w_bytes;
    const uint32_t bar_wfull = sm.bar(B_W_FULL), bar_wempty = sm.bar(B_W_EMPTY);
    const uint32_t bar_tfull = sm.bar(B_T_FULL), bar_tempty = sm.bar(B_T_EMPTY);
    const bool split = p.prec == 3;
    const uint32_t wlo_d = (uint32_t)p.max_wgroup >> 4;
    Prof pf(sm.prof(2), p.prof != nullptr);  // 0 wait A operand, 1 wait weights, 2 wait TMEM, 3 issue
    for (int64_t tile = blockIdx.x; tile < n_tiles; tile += gridDim.x) {
        SumStep nx = load_sum_step(p.steps, sum_steps, 0);
        for (int si = 0; si < n_sum; ++si) {
            const SumStep st = nx;
            if (si + 1 < n_sum) nx = load_sum_step(p.steps, sum_steps, si + 1);
            const bool bot = st.type == 1;
            const int G = st.n_groups, ksteps = st.kpad / 16;
            uint32_t a_addr;
            if (bot) {
                const int ab = (int)(kb % Cols<LTC>::NAB);
                bar_wait(sm.bar(B_B_FULL + ab), (kb / Cols<LTC>::NAB) & 1u);
                a_addr = smem_u32(sm.bimg(ab));
            } else {
                bar_wait(sm.bar(B_U_FULL), ku & 1u);
                a_addr = smem_u32(sm.uimg());
            }
            pf.mark(0);
            const uint64_t a_desc = a_hi_bits | (uint64_t)((a_addr >> 4) & 0x3FFFu);
            const uint32_t a_lo_d = ((uint32_t)(bot ? p.bimg_bytes : p.uimg_bytes) / 2) >> 4;
            const uint32_t ka_d = (2 * lbo_a) >> 4;
#if EPI_SHARE || R2_MMA_PERGROUP
            // per group: wait only for this group's accumulator, so group g+1's
            // chain starts while the epilogue still drains the other buffer
            for (int gi = 0; gi < G; ++gi) {
                const int b = gi & 1;
                const GroupInfo gr = group_info(st, gi);
                uint32_t wsl = 0;
                pf.mark(3);
                if (gr.ns > 0) {
                    wsl = w_idx;
                    bar_wait(bar_wfull + 8u * w_idx, w_ph);
                    if (++w_idx == n_w) {
                        w_idx = 0;
                        w_ph ^= 1u;
                    }
                }
                pf.mark(1);
                bar_wait(bar_tempty + 8u * b, (tp & 1u) ^ 1u);
                pf.mark(2);
                tc_fence_after();
                if (lane == 0) {
                    const uint32_t lbo_b = (uint32_t)gr.ncol * 16;
                    const uint64_t w_desc =
                        desc_hi(lbo_b, 128) | (uint64_t)(((wbase + wsl * wstride) >> 4) & 0x3FFFu);
                    const uint32_t kw_d = (2 * lbo_b) >> 4;
                    const uint32_t idesc = (1u << 4) | ((uint32_t)(gr.ncol >> 3) << 17) | ((uint32_t)(RT >> 4) << 24);
                    const uint32_t d = tmem + (b ? (uint32_t)Cols<LTC>::A : 0u);
#ifndef R2_KO_MMA
                    if (gr.ns > 0)
                        for (int kk = 0; kk < ksteps; ++kk) {
                            const uint64_t ad = a_desc + kk * ka_d, wd = w_desc + kk * kw_d;
                            umma_f16(d, ad, wd, idesc, kk > 0);
                            if (split) {
                                umma_f16(d, ad + a_lo_d, wd, idesc, 1);
                                umma_f16(d, ad, wd + wlo_d, idesc, 1);
                            }
                        }
#endif
#ifdef R2_TRACE
                    pf.mark(4);
#endif
                    umma_commit(bar_tfull + 8u * b);
#ifdef R2_TRACE
                    pf.mark(5);
#endif
#if !R2_EPI_RELEASE
                    if (gr.ns > 0) umma_commit(bar_wempty + 8u * wsl);
#endif
#ifdef R2_TRACE
                    pf.mark(6);
#endif
                }
                __syncwarp();
                if (b) ++tp;
            }
#else
            for (int gp = 0; gp < G; gp += 2, ++tp) {
                GroupInfo gr[2] = {group_info(st, gp), group_info(st, gp + 1)};
                uint32_t wsl[2] = {0, 0};
                pf.mark(3);
#pragma unroll
                for (int b = 0; b < 2; ++b) {
                    if (gr[b].ns > 0) {
                        wsl[b] = w_idx;
                        bar_wait(bar_wfull + 8u * w_idx, w_ph);
                        if (++w_idx == n_w) {
                            w_idx = 0;
                            w_ph ^= 1u;
                        }
                    }
                }
                pf.mark(1);
                bar_wait(bar_tempty, (tp & 1u) ^ 1u);
                bar_wait(bar_tempty + 8u, (tp & 1u) ^ 1u);
                pf.mark(2);
                tc_fence_after();
                if (lane == 0) {
                    uint64_t w_desc[2];
                    uint32_t idesc[2], kw_d[2];
#pragma unroll
                    for (int b = 0; b < 2; ++b) {
                        const uint32_t lbo_b = (uint32_t)gr[b].ncol * 16;
                        w_desc[b] = desc_hi(lbo_b, 128) | (uint64_t)(((wbase + wsl[b] * wstride) >> 4) & 0x3FFFu);
                        kw_d[b] = (2 * lbo_b) >> 4;
                        idesc[b] = (1u << 4) | ((uint32_t)(gr[b].ncol >> 3) << 17) | ((uint32_t)(RT >> 4) << 24);
                    }
#ifndef R2_KO_MMA  // knockout (wrong results): commits only, no tensor-core work
#if R2_MMA_INTERLEAVE
                    for (int kk = 0; kk < ksteps; ++kk) {
#pragma unroll
                        for (int b = 0; b < 2; ++b) {
#else
                    // each accumulator's K-steps back to back: chained MMAs into
                    // one accumulator pipeline, while an MMA whose accumulator
                    // was last written by an earlier, non-adjacent MMA waits for
                    // it (scripts/micro/umma_issue.cu: 160 vs 294 cycles per MMA
                    // for two accumulators, K-steps consecutive vs interleaved)
#pragma unroll
                    for (int b = 0; b < 2; ++b) {
                        for (int kk = 0; kk < ksteps; ++kk) {
#endif
                            if (gr[b].ns > 0) {
                                const uint32_t d = tmem + (b ? (uint32_t)Cols<LTC>::A : 0u);
                                const uint64_t ad = a_desc + kk * ka_d, wd = w_desc[b] + kk * kw_d[b];
                                umma_f16(d, ad, wd, idesc[b], kk > 0);
                                if (split) {
                                    umma_f16(d, ad + a_lo_d, wd, idesc[b], 1);
                                    umma_f16(d, ad, wd + wlo_d, idesc[b], 1);
                                }
                            }
                        }
                    }
#endif
                    umma_commit(bar_tfull);
                    umma_commit(bar_tfull + 8u);
#pragma unroll
                    for (int b = 0; b < 2; ++b)
                        if (gr[b].ns > 0) umma_commit(bar_wempty + 8u * wsl[b]);
                }
                __syncwarp();
            }
#endif
#if !R2_EPI_RELEASE
            if (lane == 0) umma_commit(sm.bar(bot ? B_B_EMPTY + (int)(kb % Cols<LTC>::NAB) : B_U_EMPTY));
            __syncwarp();
#endif
            if (bot) ++kb;
            else ++ku;
            pf.mark(3);
        }
    }
}

// ============================================================== EPILOGUE
// Thread = sample m = TMEM lane.  TMEM columns: [0, NACC GC) accumulators,
// then D activation slots of S columns, then C root accumulators.  Widths
// are template parameters (I: leaf regions, S: sum regions), so a sum's
// stage-2 contraction is straight-line code.

template <int W>
__device__ __forceinline__ void ld_unit_any(uint32_t taddr, float (&t)[W]) {
#pragma unroll
    for (int c = 0; c + 8 <= W; c += 8) tmem_ld8(taddr + c, t + c);
    if constexpr (W % 8) tmem_ld4(taddr + (W / 8) * 8, t + (W / 8) * 8);
}
// One sum step's groups: out_s = shift + lg2(sum_i ea_i T[s, i]) - k_s.
// Group gi lives in accumulator gi & 1; its sums are read one at a time,
// double-buffered (the next sum's tcgen05.ld is in flight while this sum's
// FFMA2s run; tcgen05.wait::ld then covers it).
// partial dot product of U columns against ea[off .. off + U)
template <int U, int NA>
__device__ __forceinline__ float dot_part(const float (&ea)[NA], int off, const float (&t)[U]) {
    float2 p0 = make_float2(0.f, 0.f), p1 = make_float2(0.f, 0.f);
#pragma unroll
    for (int i = 0; i + 4 <= U; i += 4) {
        p0 = __ffma2_rn(make_float2(ea[off + i], ea[off + i + 1]), make_float2(t[i], t[i + 1]), p0);
        p1 = __ffma2_rn(make_float2(ea[off + i + 2], ea[off + i + 3]), make_float2(t[i + 2], t[i + 3]),
                        p1);
    }
    return (p0.x + p0.y) + (p1.x + p1.y);
}
// W columns of one TMEM lane (W a multiple of 4): x16 / x8 / x4 loads
template <int W>
__device__ __forceinline__ void ld_cols(uint32_t taddr, float *t) {
#pragma unroll
    for (int c = 0; c + 16 <= W; c += 16) tmem_ld16(taddr + c, t + c);
    if constexpr (W % 16 >= 8) tmem_ld8(taddr + (W / 16) * 16, t + (W / 16) * 16);
    if constexpr (W % 8) tmem_ld4(taddr + (W / 8) * 8, t + (W / 8) * 8);
}
// sum_i ea_i t_i with four FFMA2 chains (eight partial sums)
template <int NA>
__device__ __forceinline__ float dot4(const float (&ea)[NA], const float *t) {
    float2 q[4] = {make_float2(0.f, 0.f), make_float2(0.f, 0.f), make_float2(0.f, 0.f),
                   make_float2(0.f, 0.f)};
#pragma unroll
    for (int i = 0; i + 2 <= NA; i += 2)
        q[(i / 2) & 3] = __ffma2_rn(make_float2(ea[i], ea[i + 1]), make_float2(t[i], t[i + 1]), q[(i / 2) & 3]);
    return ((q[0].x + q[0].y) + (q[1].x + q[1].y)) + ((q[2].x + q[2].y) + (q[3].x + q[3].y));
}

// R2_EPI_RELEASE: lane 0 of the lane-quarter-0 warp draining a group
// releases that group's weight slot once it has seen the group's T_FULL
// (the MMAs that read the slot are complete), and the warp draining the
// step's last group releases the step's operand image (rel_bar); wslot is
// the weight-ring position of the step's first non-empty group
template <int NA, bool ROOT, bool LTC>
__device__ __forceinline__ void sum_groups(const R2Params &p, const Smem &sm, const SumStep &st,
                                           const float (&ear)[NA], float shift, uint32_t lane_base,
                                           uint32_t out_col, uint32_t col_root, uint32_t &tp,
                                           Prof &pf, int h, uint32_t &wslot, uint32_t rel_bar,
                                           bool releaser) {
    static_assert(NA % 4 == 0, "region width");
    constexpr int PB = NA >= EPI_COLS ? 1 : EPI_COLS / NA;  // sums per TMEM batch
    const float *ks = p.fparams + st.blk_off;
    auto fin = [&](int s, float a, float k) {
        const float val = shift + lg2(a) - k;
        if constexpr (ROOT) {
            const uint32_t c = col_root + (uint32_t)__ldg(p.root_map + s);
            float r;
            tmem_ld1(lane_base + c, r);
            tmem_wait_ld();
            tmem_st1(lane_base + c, lse2(r, val));
        } else {
            tmem_st1(lane_base + out_col + s, val);
        }
    };
    const int G = st.n_groups;
#if EPI_SHARE
    // both warps of the lane quarter take every group, alternating its sums
    constexpr int QB = NA >= EPI_COLS / 2 ? 1 : EPI_COLS / 2 / NA;  // own sums per TMEM batch
    for (int gi = 0; gi < G; ++gi) {
        const int b = gi & 1;
        const GroupInfo gr = group_info(st, gi);
        pf.mark(3);
        bar_wait(sm.bar(B_T_FULL + b), (tp & 1u));
        pf.mark(2);
        tc_fence_after();
        const uint32_t acc = lane_base + (b ? (uint32_t)Cols<LTC>::A : 0u);
        const int ns = gr.ns;
        const int mine = ns > h ? (ns - h + 1) / 2 : 0;  // this warp's sums: h, h + 2, ...
        for (int k0 = 0; k0 < mine; k0 += QB) {
            float t[QB * NA], kv[QB];
#pragma unroll
            for (int k = 0; k < QB; ++k) {
                const int sl = h + 2 * (k0 + k);
                if (k0 + k < mine) ld_cols<NA>(acc + (uint32_t)(sl * NA), t + k * NA);
                kv[k] = k0 + k < mine ? __ldg(ks + gr.s0 + sl) : 0.f;
            }
            tmem_wait_ld();
            if (k0 + QB >= mine) {
                tc_fence_before();
                bar_arrive(sm.bar(B_T_EMPTY + b));
            }
            float val[QB];
#pragma unroll
            for (int k = 0; k < QB; ++k) val[k] = dot4(ear, t + k * NA);
#pragma unroll
            for (int k = 0; k < QB; ++k)
                if (k0 + k < mine) fin(gr.s0 + h + 2 * (k0 + k), val[k], kv[k]);
        }
        if (mine == 0) {
            tc_fence_before();
            bar_arrive(sm.bar(B_T_EMPTY + b));
        }
        if (b) ++tp;
    }
    return;
#endif
#if R2_EPI_RELEASE
    uint32_t wpos = wslot;  // ring position of group gi's weights (non-empty groups only)
    const uint32_t n_w = (uint32_t)p.n_w;
#endif
    for (int gi = 0; gi < G; ++gi) {
#if R2_EPI_RELEASE
        const GroupInfo gr = group_info(st, gi);
        const uint32_t my_w = wpos;
        if (gr.ns > 0 && ++wpos == n_w) wpos = 0;
        if ((gi & 1) != h) continue;  // this warp's accumulator: groups of parity h
#else
        if ((gi & 1) != h) continue;
        const GroupInfo gr = group_info(st, gi);
#endif
        const int b = gi & 1;
        pf.mark(3);
        bar_wait(sm.bar(B_T_FULL + b), (tp & 1u));
        pf.mark(2);
        tc_fence_after();
#if R2_EPI_RELEASE
        if (releaser) {
            if (gr.ns > 0) bar_arrive(sm.bar(B_W_EMPTY) + 8u * my_w);
            if (gi == G - 1) bar_arrive(rel_bar);
        }
#endif
        const uint32_t acc = lane_base + (b ? (uint32_t)Cols<LTC>::A : 0u);
        const int ns = gr.ns;
        // batches of PB sums (one tcgen05.ld of PB * NA <= 80 columns, one
        // wait): the sums' dot products are independent chains the scheduler
        // interleaves (a lone warp's per-sum chain -- FFMA2s, reduction, lg2,
        // subtract, store -- measured ~190 cycles; scripts/micro/epi_sum.cu)
        for (int sl = 0; sl < ns; sl += PB) {
            float t[PB * NA], kv[PB];
#ifdef R2_KO_TLD  // knockout (wrong results): no accumulator reads
#pragma unroll
            for (int k = 0; k < PB * NA; ++k) t[k] = __int_as_float(acc + k);
#else
            ld_cols<PB * NA>(acc + (uint32_t)(sl * NA), t);
#endif
#pragma unroll
            for (int k = 0; k < PB; ++k)  // the sums' scale exponents, in flight with the TMEM batch
                kv[k] = sl + k < ns ? __ldg(ks + gr.s0 + sl + k) : 0.f;
            tmem_wait_ld();
#ifdef R2_TRACE
            pf.mark(6);
#endif
            if (sl + PB >= ns) {
                tc_fence_before();
                bar_arrive(sm.bar(B_T_EMPTY + b));  // all of this group's columns are in registers
            }
            float val[PB];
#ifdef R2_KO_EPI  // knockout (wrong results): no stage-2 dot products
#pragma unroll
            for (int k = 0; k < PB; ++k) val[k] = t[k * NA] + ear[k];
#else
#pragma unroll
            for (int k = 0; k < PB; ++k) val[k] = dot4(ear, t + k * NA);
#endif
#pragma unroll
            for (int k = 0; k < PB; ++k)
                if (sl + k < ns) fin(gr.s0 + sl + k, val[k], kv[k]);
#ifdef R2_TRACE
            pf.mark(7);
#endif
        }
        if (ns == 0) {
            tc_fence_before();
            bar_arrive(sm.bar(B_T_EMPTY + b));
        }
        ++tp;
    }
#if R2_EPI_RELEASE
    wslot = wpos;
#endif
}

// ============================================================== LEAF on tensor cores (LTC)
// Gaussian leaf region (log2 units): L[m, i] = sum_v
// c_vi - (a_vi x_mv - b_vi)^2.  Expanded around a per-variable centre M_v
// (x~ = x - M_v, b~ = b - a M_v) it is one GEMM over the features
//   F[m] = (x~_0^2, x~_0, x~_1^2, x~_1, ..., 1)            joint
//   F[m] = (x~_0^2, x~_0, ..., z_0, z_1, ...)               marginal (z_v = x_v observed;
//                                                            a missing x_v has x~ = 0)
// against P = (-a^2, 2 a b~, ..., c - b~^2) (layered.cpp build_rat2).  The
// operands are split hi/lo in f16 (F = F_h + F_l, P = P_h + P_l) and
// L = F_h P_h + F_h P_l + F_l P_h accumulates in fp32 in TMEM: about 2^-21
// relative per term, fp32-class like the FMA leaves it replaces.  A
// sample whose |x~| exceeds 240 (f16 range of x~^2) or is infinite gets a NaN
// shift, hence NaN outputs, which the certification recomputes in v1.
//
// Leaf warps (thread = sample m = TMEM lane): per region l, read back
// L(l-1), build F(l) (the single feature image is free once L(l-1) is
// complete), hand it to the leaf MMA warp, then the shift / exps of l-1
// while the tensor core computes L(l).
template <int I, bool MARG>
__device__ void leaf_tc_role(const R2Params &p, const Smem &sm, const int32_t *leaf_steps,
                             int n_leaf, uint32_t tmem, int warp, int lane) {
    static_assert(I % 8 == 0, "leaf width");
    constexpr int NAB2 = Cols<true>::NAB;
    const int m = warp * 32 + lane;
    const uint32_t lacc = tmem + ((uint32_t)(warp * 32) << 16) + (uint32_t)Cols<true>::L;
    const int64_t n_tiles = (p.n + RT - 1) / RT;
    uint8_t *fh = sm.fimg();
    uint8_t *fl = fh + p.f_bytes;
    const int nq = p.lvp >> 2;
    const int zcol = 2 * p.lvp;
    const uint32_t n_in = (uint32_t)p.n_in;
    uint32_t li = 0, s = 0, sph = 0;
    bool bad_prev = false;
    float L[I];
    Prof pf(sm.prof(0), p.prof != nullptr);  // 0 wait input, 1 build F, 2 wait L, 3 wait output slot, 4 exps + write
    // shift / exps of region lj (values in L) into its left / right slot
    auto exps = [&](uint32_t lj, bool bad) {
        const bool side_b = (lj & 1u) != 0;
        const uint32_t j = lj >> 1;
        float h = L[0];
#pragma unroll
        for (int i = 1; i < I; ++i) h = maxnan(h, L[i]);
        if (bad) h = CUDART_NAN_F;
        const int ab = (int)(j % NAB2);
        const uint32_t ph = (j / NAB2) & 1u;
        bar_wait(sm.bar(B_A_EMPTY + ab), ph ^ 1u);
        if (side_b) bar_wait(sm.bar(B_B_EMPTY + ab), ph ^ 1u);
        pf.mark(3);
        if (!side_b) {
            float *ea = sm.ea(ab);
            const float hc = fmaxf(h, -1e30f);
#pragma unroll
            for (int i = 0; i < I; ++i) ea[i * RT + m] = ex2(L[i] - hc);
            sm.ha(ab)[m] = h;
            bar_arrive(sm.bar(B_A_FULL + ab));
        } else {
            uint8_t *img = sm.bimg(ab);
            const float hc = fmaxf(h, -1e30f) - EB_SHIFT;
#pragma unroll
            for (int i = 0; i < I; i += 8)
                *reinterpret_cast<uint4 *>(img + img_off(m, i)) =
                    make_uint4(pack_h2(ex2(L[i] - hc), ex2(L[i + 1] - hc)),
                               pack_h2(ex2(L[i + 2] - hc), ex2(L[i + 3] - hc)),
                               pack_h2(ex2(L[i + 4] - hc), ex2(L[i + 5] - hc)),
                               pack_h2(ex2(L[i + 6] - hc), ex2(L[i + 7] - hc)));
            sm.hb(ab)[m] = h - EB_SHIFT;
            fence_async_smem();
            bar_arrive(sm.bar(B_B_FULL + ab));
        }
        pf.mark(4);
    };
    auto read_l = [&](uint32_t lj) {
        bar_wait(sm.bar(B_LT_FULL), lj & 1u);
        tc_fence_after();
        ld_cols<I>(lacc, L);
        tmem_wait_ld();
        pf.mark(2);
    };
    for (int64_t tile = blockIdx.x; tile < n_tiles; tile += gridDim.x) {
        for (int l = 0; l < n_leaf; ++l, ++li) {
            const int V = __ldg(&p.steps[__ldg(leaf_steps + l)].n_vars);
            bar_wait(sm.bar(B_IN_FULL + (int)s), sph);
            pf.mark(0);
            if (li > 0) read_l(li - 1);  // also: the feature image is free again
            const float *xs = sm.in_x((int)s);
            const float *Mv = sm.in_prm((int)s);
            float amax = 0.f;
            for (int c = 0; c < nq; ++c) {
                const float4 M4 = *reinterpret_cast<const float4 *>(Mv + 4 * c);
                const float mm[4] = {M4.x, M4.y, M4.z, M4.w};
                uint32_t hw[4], lw[4];
                float zf[4];
#pragma unroll
                for (int k = 0; k < 4; ++k) {
                    const int v = 4 * c + k;
                    float xt = (v < V ? xs[v * RT + m] : mm[k]) - mm[k];
                    float z = v < V ? 1.f : 0.f;
                    if constexpr (MARG) {
                        const bool nan = xt != xt;
                        xt = nan ? 0.f : xt;
                        z = nan ? 0.f : z;
                    }
                    amax = fmaxf(amax, fabsf(xt));
                    const float q = xt * xt;
                    hw[k] = pack_h2(q, xt);
                    const float2 hf = __half22float2(*reinterpret_cast<const __half2 *>(&hw[k]));
                    lw[k] = pack_h2(q - hf.x, xt - hf.y);
                    zf[k] = z;
                }
                const uint32_t o = img_off(m, 8 * c);
                *reinterpret_cast<uint4 *>(fh + o) = make_uint4(hw[0], hw[1], hw[2], hw[3]);
                *reinterpret_cast<uint4 *>(fl + o) = make_uint4(lw[0], lw[1], lw[2], lw[3]);
                if constexpr (MARG)
                    *reinterpret_cast<uint2 *>(fh + img_off(m, zcol + 4 * c)) =
                        make_uint2(pack_h2(zf[0], zf[1]), pack_h2(zf[2], zf[3]));
            }
            const bool bad = !(amax <= 240.f);
            fence_async_smem();  // the feature image is read by the tensor core (async proxy)
            tc_fence_before();   // ... and the tcgen05.ld of L(l-1) is complete
            bar_arrive(sm.bar(B_F_FULL));
            pf.mark(1);
            if (li > 0) exps(li - 1, bad_prev);
            bad_prev = bad;
            if (++s == n_in) {
                s = 0;
                sph ^= 1u;
            }
        }
    }
    if (li > 0) {
        read_l(li - 1);
        exps(li - 1, bad_prev);
    }
}

// Leaf MMA warp (LTC): L = F_h P_h + F_h P_l + F_l P_h (M = 128, N = 48,
// K = kl) into the leaf accumulator; the commit releases the input slot
// (the parameter image) and signals the leaf warps.  A second issuing warp
// keeps the leaf GEMMs off the sum-layer MMA warp's chain.
template <bool MARG>
__device__ void leaf_mma_role(const R2Params &p, const Smem &sm, int n_leaf, uint32_t tmem,
                              int lane) {
    constexpr uint32_t NL = R2T_COLS_L;
    const int64_t n_tiles = (p.n + RT - 1) / RT;
    const uint32_t d = tmem + (uint32_t)Cols<true>::L;
    const uint32_t idesc = (1u << 4) | ((NL >> 3) << 17) | ((uint32_t)(RT >> 4) << 24);
    const uint64_t a_hi = desc_hi(RT * 16, 128), b_hi = desc_hi(NL * 16, 128);
    const int kl = MARG ? p.kl_m : p.kl_j;
    const int ks = kl >> 4, ks_lo = (2 * p.lvp + 15) >> 4;
    const uint32_t ka_d = (2 * RT * 16) >> 4, kb_d = (2 * NL * 16) >> 4;
    const uint32_t fa = smem_u32(sm.fimg()), fl = fa + (uint32_t)p.f_bytes;
    const uint32_t pbytes = NL * (uint32_t)kl * 2;
    const uint32_t n_in = (uint32_t)p.n_in;
    uint32_t li = 0, s = 0, sph = 0;
    for (int64_t tile = blockIdx.x; tile < n_tiles; tile += gridDim.x) {
        for (int l = 0; l < n_leaf; ++l, ++li) {
            bar_wait(sm.bar(B_F_FULL), li & 1u);
            bar_wait(sm.bar(B_IN_FULL + (int)s), sph);  // the parameter image has landed
            tc_fence_after();
            if (lane == 0) {
                const uint32_t pa = smem_u32(sm.in_pimg((int)s)), pl = pa + pbytes;
                const uint64_t A = a_hi | (uint64_t)((fa >> 4) & 0x3FFFu);
                const uint64_t Al = a_hi | (uint64_t)((fl >> 4) & 0x3FFFu);
                const uint64_t B = b_hi | (uint64_t)((pa >> 4) & 0x3FFFu);
                const uint64_t Bl = b_hi | (uint64_t)((pl >> 4) & 0x3FFFu);
                for (int kk = 0; kk < ks; ++kk) umma_f16(d, A + kk * ka_d, B + kk * kb_d, idesc, kk > 0);
                for (int kk = 0; kk < ks; ++kk) umma_f16(d, A + kk * ka_d, Bl + kk * kb_d, idesc, 1);
                for (int kk = 0; kk < ks_lo; ++kk) umma_f16(d, Al + kk * ka_d, B + kk * kb_d, idesc, 1);
                umma_commit(sm.bar(B_LT_FULL));
                umma_commit(sm.bar(B_IN_EMPTY + (int)s));
            }
            __syncwarp();
            if (++s == n_in) {
                s = 0;
                sph ^= 1u;
            }
        }
    }
}

template <int I, int S, bool MARG, bool LTC>
__device__ void epilogue_role(const R2Params &p, const Smem &sm, const int32_t *sum_steps,
                              int n_sum, uint32_t tmem, int warp, int lane) {
    const int qd = warp & 3;
    const int h = (warp - W_EPI0) >> 2;  // 0: groups in accumulator A, 1: in accumulator B
    const int m = qd * 32 + lane;
    const uint32_t lane_base = tmem + ((uint32_t)(qd * 32) << 16);
    const uint32_t col_slots = (uint32_t)Cols<LTC>::SLOTS;
    // the two warps of a lane quarter exchange activation slots / root
    // columns through TMEM: wait for own stores, then a 64-thread barrier
    auto pair_sync = [&]() {
        tmem_wait_st();
        tc_fence_before();
        asm volatile("bar.sync %0, 64;" ::"r"(1 + qd) : "memory");
        tc_fence_after();
    };
    const uint32_t col_root = col_slots + (uint32_t)(p.D * S);
    const int64_t n_tiles = (p.n + RT - 1) / RT;
    uint32_t kb = 0, ku = 0, tp = 0;
    uint32_t wslot = 0;                          // weight-ring position (R2_EPI_RELEASE)
    const bool releaser = qd == 0 && lane == 0;  // releases slots for this warp's groups
    const int part_u = p.uimg_bytes / 2;
    constexpr int SU = S > 0 ? S : 4;
    Prof pf(sm.prof(1), p.prof != nullptr);  // 0 wait leaf outputs, 1 UP phase 1, 2 wait TMEM full, 3 sums, 4 tile I/O, 5 step setup
    for (int64_t tile = blockIdx.x; tile < n_tiles; tile += gridDim.x) {
        if (h == 0)
            for (int c = 0; c < p.C; ++c) tmem_st1(lane_base + col_root + c, -CUDART_INF_F);
        pair_sync();
        SumStep nx = load_sum_step(p.steps, sum_steps, 0);
        for (int si = 0; si < n_sum; ++si) {
            const SumStep es = nx;
            if (si + 1 < n_sum) nx = load_sum_step(p.steps, sum_steps, si + 1);
            pf.mark(5);
            const uint32_t out_col = col_slots + (uint32_t)((es.slot_out - 1) * S);
            if (es.type == 1) {
                // BOT: ea from leaf group 0, hb from leaf group 1
                const int ab = (int)(kb % Cols<LTC>::NAB);
                const uint32_t ph = (kb / Cols<LTC>::NAB) & 1u;
                bar_wait(sm.bar(B_A_FULL + ab), ph);
                bar_wait(sm.bar(B_B_FULL + ab), ph);
                pf.mark(0);
                const float *ea = sm.ea(ab);
                float ear[I];
#pragma unroll
                for (int i = 0; i < I; ++i) ear[i] = ea[i * RT + m];
                const float shift = sm.ha(ab)[m] + sm.hb(ab)[m];
                bar_arrive(sm.bar(B_A_EMPTY + ab));
                const uint32_t rel_b = sm.bar(B_B_EMPTY + ab);  // the B image, after the step's MMAs
                ++kb;
                if (es.root) sum_groups<I, true, LTC>(p, sm, es, ear, shift, lane_base, out_col, col_root, tp, pf, h, wslot, rel_b, releaser);
                else sum_groups<I, false, LTC>(p, sm, es, ear, shift, lane_base, out_col, col_root, tp, pf, h, wslot, rel_b, releaser);
            } else {
                // UP: children in activation slots; B side -> f16 image, A side -> registers
                float vb[SU], ear[SU];
                pair_sync();  // the children's sums were written by both warps
                ld_unit_any<SU>(lane_base + col_slots + (uint32_t)((es.slot_b - 1) * S), vb);
                ld_unit_any<SU>(lane_base + col_slots + (uint32_t)((es.slot_a - 1) * S), ear);
                tmem_wait_ld();
                float hb = vb[0], ha = ear[0];
#pragma unroll
                for (int i = 1; i < SU; ++i) {
                    hb = maxnan(hb, vb[i]);
                    ha = maxnan(ha, ear[i]);
                }
                if (h == R2_UPIMG_H) {  // one warp of the pair writes the B-side operand image
                    bar_wait(sm.bar(B_U_EMPTY), (ku & 1u) ^ 1u);
                    uint8_t *img = sm.uimg();
                    const float hc = fmaxf(hb, -1e30f) - EB_SHIFT;
#pragma unroll
                    for (int i = 0; i < SU; i += 2) {
                        const float e0 = ex2(vb[i] - hc), e1 = i + 1 < SU ? ex2(vb[i + 1] - hc) : 0.f;
                        const uint32_t o = img_off(m, i);
                        if (p.prec == 3) {
                            uint32_t hi, lo;
                            split_h2(e0, e1, hi, lo);
                            *reinterpret_cast<uint32_t *>(img + o) = hi;
                            *reinterpret_cast<uint32_t *>(img + part_u + o) = lo;
                        } else {
                            *reinterpret_cast<uint32_t *>(img + o) = pack_h2(e0, e1);
                        }
                    }
                    fence_async_smem();
                    bar_arrive(sm.bar(B_U_FULL));
                }
                ++ku;
                const float hac = fmaxf(ha, -1e30f);
#pragma unroll
                for (int i = 0; i < SU; ++i) ear[i] = ex2(ear[i] - hac);
                const float shift = ha + hb - EB_SHIFT;
                pf.mark(1);
                if (es.root) sum_groups<SU, true, LTC>(p, sm, es, ear, shift, lane_base, out_col, col_root, tp, pf, h, wslot, sm.bar(B_U_EMPTY), releaser);
                else sum_groups<SU, false, LTC>(p, sm, es, ear, shift, lane_base, out_col, col_root, tp, pf, h, wslot, sm.bar(B_U_EMPTY), releaser);
            }
            tmem_wait_st();
        }
        pf.mark(3);
        pair_sync();  // root columns were accumulated by both warps
        if (h == 1) continue;
        // ---- outputs of the tile (the TMEM loads stay warp-converged)
        const int64_t row = tile * RT + m;
        int best = -1;
        float bv = -CUDART_INF_F;
        bool cert = true;
        for (int c = 0; c < p.C; ++c) {
            float r;
            tmem_ld1(lane_base + col_root + c, r);
            tmem_wait_ld();
            const float v = r * 0.6931471805599453f;
            if (row < p.n) p.out[row * p.C + c] = v;
            if (!(v != v) && (best < 0 || v > bv)) {
                best = c;
                bv = v;
            }
            // single-pass error bound inside the tolerance? (NaN / inf
            // results are the same in both precisions)
            const float av = fabsf(v);
            if (av < CUDART_INF_F && !(p.cert_err <= p.cert_tol * fmaxf(1.f, av - p.cert_err)))
                cert = false;
            // tensor-core leaves: NaN marks an input outside the split operands'
            // range (or a NaN input, recomputed alike)
            if (LTC && v != v) cert = false;
        }
        if (row < p.n && p.argmax) p.argmax[row] = best;
        if (row < p.n && p.flag_count && !cert) p.flag_idx[atomicAdd(p.flag_count, 1)] = p.row0 + row;
        pf.mark(4);
    }
}

template <int I, int S, bool MARG, bool LTC>
__global__ void __launch_bounds__(NTHREADS, 1)
    rat2_kernel(const R2Params p, const int32_t *__restrict__ leaf_steps, int n_leaf,
                const int32_t *__restrict__ sum_steps, int n_sum) {
    extern __shared__ __align__(1024) uint8_t smem_raw[];
    // realign with pointer arithmetic on the __shared__ array (a round trip
    // through uintptr_t would make every access a generic LD/ST)
    uint8_t *base = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
    const Smem sm(base, p);
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    uint32_t *tmem_slot = reinterpret_cast<uint32_t *>(base + p.off_bar + 8 * B_COUNT);
    if (warp == W_MMA) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(
            smem_u32(tmem_slot)));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    if (tid == 0) {
        for (int i = 0; i < 4; ++i) {
            bar_init(sm.bar(B_IN_FULL + i), 1);
            // the warps of one leaf group (LTC: the leaf MMA's commit)
            bar_init(sm.bar(B_IN_EMPTY + i), LTC ? 1 : WPG);
        }
        for (int i = 0; i < 8; ++i) {
            bar_init(sm.bar(B_W_FULL + i), 1);
            bar_init(sm.bar(B_W_EMPTY + i), 1);
        }
        for (int i = 0; i < Cols<LTC>::NAB; ++i) {
            // the threads of one leaf group (LTC: the 128 leaf threads, one per sample)
            bar_init(sm.bar(B_A_FULL + i), LTC ? 128 : WPG * 32);
            bar_init(sm.bar(B_A_EMPTY + i), 256);  // both epilogue warps of each quarter
            bar_init(sm.bar(B_B_FULL + i), LTC ? 128 : WPG * 32);
            bar_init(sm.bar(B_B_EMPTY + i), 1);
        }
        for (int i = 0; i < 2; ++i) {
            bar_init(sm.bar(B_T_FULL + i), 1);
            bar_init(sm.bar(B_T_EMPTY + i), EPI_SHARE ? 256 : 128);  // epilogue threads draining it
        }
        bar_init(sm.bar(B_U_FULL), 128);
        bar_init(sm.bar(B_U_EMPTY), 1);
        bar_init(sm.bar(B_F_FULL), 128);
        bar_init(sm.bar(B_LT_FULL), 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        for (int k = 0; k < 32; ++k) sm.prof(0)[k] = 0;
    }
    // zero the operand images once (the K padding columns stay zero)
    for (int i = tid * 16; i < Cols<LTC>::NAB * p.bimg_bytes + p.uimg_bytes; i += NTHREADS * 16)
        *reinterpret_cast<uint4 *>(base + p.off_bimg + i) = make_uint4(0, 0, 0, 0);
    if constexpr (LTC) {
        static_assert(NLG == 1, "tensor-core leaves: one leaf warpgroup (thread = sample)");
        // feature image: zero (K padding, lo part of the constant columns),
        // joint: the constant column 2 lvp = 1
        for (int i = tid * 16; i < 2 * p.f_bytes; i += NTHREADS * 16)
            *reinterpret_cast<uint4 *>(sm.fimg() + i) = make_uint4(0, 0, 0, 0);
        __syncthreads();
        if (!MARG && tid < RT)
            *reinterpret_cast<uint16_t *>(sm.fimg() + img_off(tid, 2 * p.lvp)) = 0x3C00u;  // f16 1.0
    }
    fence_async_smem();
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem = *tmem_slot;

    // launch: 128 registers per thread (16 warps); leaf 152, epilogue 152,
    // producers / MMA 56: 152 + 2 * 152 + 56 = 512 per SMSP lane
    if (warp >= W_PROD) asm volatile("setmaxnreg.dec.sync.aligned.u32 %0;" ::"n"(REG_PROD));
    else if (warp >= W_EPI0) asm volatile("setmaxnreg.inc.sync.aligned.u32 %0;" ::"n"(REG_EPI));
    else if (REG_LEAF > LAUNCH_REGS)
        asm volatile("setmaxnreg.inc.sync.aligned.u32 %0;" ::"n"(REG_LEAF));
    if (warp < W_EPI0) {
        if constexpr (LTC) leaf_tc_role<I, MARG>(p, sm, leaf_steps, n_leaf, tmem, warp, lane);
        else leaf_role<I / 4, MARG>(p, sm, leaf_steps, n_leaf, warp, lane);
    } else if (warp < W_PROD) {
        epilogue_role<I, S, MARG, LTC>(p, sm, sum_steps, n_sum, tmem, warp, lane);
    } else if (warp == W_PROD) {
        leaf_producer_role<LTC, MARG>(p, sm, leaf_steps, n_leaf, lane);
    } else if (warp == W_MMA) {
        mma_role<LTC>(p, sm, sum_steps, n_sum, tmem, lane);
    } else if (warp == W_WPROD) {
        weight_producer_role(p, sm, sum_steps, n_sum, lane);
    } else if (LTC && warp == W_WPROD + 1) {
        leaf_mma_role<MARG>(p, sm, n_leaf, tmem, lane);
    }
    tc_fence_before();
    __syncthreads();
    if (p.prof && tid < 32) atomicAdd(p.prof + tid, sm.prof(0)[tid]);
    if (warp == W_MMA) {
        tc_fence_after();
        asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(tmem));
    }
}

}  // namespace r2

#ifdef R2_TRACE
extern "C" int spnb_r2_trace(unsigned long long *out, int max_pairs) {
    // all per-warp regions (unused entries are zero); clears them
    const int n = std::min(max_pairs, (int)r2::TRACE_N);
    cudaMemcpyFromSymbol(out, r2::g_trace, 2 * sizeof(unsigned long long) * n);
    static unsigned long long zero[2 * 4096];
    for (unsigned o = 0; o < 2 * r2::TRACE_N; o += 2 * 4096)
        cudaMemcpyToSymbol(r2::g_trace, zero, sizeof(zero), o * sizeof(unsigned long long));
    return n;
}
#endif

// (I, S) pairs with a compiled kernel instance (S = 0: no sum regions)
bool rat2_supported_shape(int I, int S) {
    static const int kShapes[][2] = {{8, 4}, {16, 8}, {40, 20}, {32, 16}, {16, 16}, {48, 24}};
    for (auto &k : kShapes)
        if (k[0] == I && (k[1] == S || (S == 0 && 2 * k[1] == I))) return true;
    return false;
}

// host: shared-memory carve-up for ring depths (n_in, n_w); returns bytes
int rat2_layout(R2Params &p, int I, int max_vars, int max_blk, int kpad_bot, int kpad_up,
                int max_wgroup, int prec, int n_in, int n_w, int lvp, int kl_j, int kl_m) {
    const int parts = prec == 3 ? 2 : 1;
    const bool ltc = lvp > 0;  // tensor-core leaves
    const int nab = ltc ? r2::Cols<true>::NAB : r2::Cols<false>::NAB;
    auto up = [](int x, int a) { return (x + a - 1) / a * a; };
    int off = 0;
    p.off_bar = off;
    off += 8 * r2::B_COUNT + 16 + 4 * 8 * 8;  // barriers, TMEM slot, profiling counters
    off = up(off, 128);
    p.n_in = n_in;
    p.in_bytes = up(max_vars * r2::RT * 4 + max_blk * 4, 128);
    p.lvp = lvp;
    p.kl_j = kl_j;
    p.kl_m = kl_m;
    p.pimg_off = p.in_bytes;
    if (ltc) p.in_bytes += 2 * R2T_COLS_L * std::max(kl_j, kl_m) * 2;  // parameter image hi + lo
    p.off_in = off;
    off += n_in * p.in_bytes;
    p.ea_bytes = up((I + 2) * r2::RT * 4, 128);
    p.off_ea = off;
    off += nab * p.ea_bytes;
    off = up(off, 1024);
    p.bimg_bytes = r2::RT * kpad_bot * 2 * parts;
    p.off_bimg = off;
    off += nab * p.bimg_bytes;
    p.uimg_bytes = r2::RT * kpad_up * 2 * parts;
    p.off_uimg = off;  // contiguous with the B images (zeroed together)
    off += p.uimg_bytes;
    off = up(off, 1024);
    p.n_w = n_w;
    p.w_bytes = up(max_wgroup * parts, 1024);
    p.off_w = off;
    off += n_w * p.w_bytes;
    p.f_bytes = ltc ? r2::RT * std::max(kl_j, kl_m) * 2 : 0;  // feature image: hi, lo
    p.off_f = off;
    off += 2 * p.f_bytes;
    p.smem_bytes = off + 1024;  // alignment slack of the dynamic base
    return p.smem_bytes;
}

cudaError_t rat2_launch(const R2Params &p, const int32_t *leaf_steps, int n_leaf,
                        const int32_t *sum_steps, int n_sum, bool marg, int grid, cudaStream_t st) {
    void (*fn)(const R2Params, const int32_t *, int, const int32_t *, int) = nullptr;
    const bool ltc = p.lvp > 0;
#define R2_CASE(I_, S_)                                                                          \
    if (p.I == I_ && (p.S == S_ || (p.S == 0 && 2 * S_ == I_)))                                  \
        fn = ltc ? (marg ? r2::rat2_kernel<I_, S_, true, true> : r2::rat2_kernel<I_, S_, false, true>) \
                 : (marg ? r2::rat2_kernel<I_, S_, true, false> : r2::rat2_kernel<I_, S_, false, false>);
    R2_CASE(8, 4) R2_CASE(16, 8) R2_CASE(40, 20) R2_CASE(32, 16) R2_CASE(16, 16) R2_CASE(48, 24)
#undef R2_CASE
    if (!fn) return cudaErrorInvalidConfiguration;
    cudaFuncAttributes fa;
    cudaError_t e = cudaFuncGetAttributes(&fa, fn);
    if (e != cudaSuccess) return e;
    if (fa.numRegs != r2::LAUNCH_REGS) return cudaErrorInvalidConfiguration;  // setmaxnreg budget
    e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, p.smem_bytes);
    if (e != cudaSuccess) return e;
    fn<<<grid, r2::NTHREADS, p.smem_bytes, st>>>(p, leaf_steps, n_leaf, sum_steps, n_sum);
    return cudaGetLastError();
}

}  // namespace spnb
