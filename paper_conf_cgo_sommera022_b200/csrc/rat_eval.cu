// rat_eval.cu -- layered RAT-SPN path for sm_100a (kernels KB + KC).
//
// For layered SPNs (RAT-SPNs, §V-B) the preparer
// (layered.cpp) turns the DAG into a per-repetition schedule of region steps.
// One persistent CTA owns a tile of 128 samples and walks the schedule:
//
//  LEAF (KB, FP32 pipe): L[i][m] = C_i - sum_v (a_iv x_mv - b_iv)^2, the log2
//       density of each of the region's I factorised Gaussians; the features
//       come from a transposed copy xT[F][N] (the LoSPN `transposed` batch
//       access, L204-227) so a region's variables are coalesced rows.
//  SUM  (KC, tensor cores): for a partition of regions A (na values a_i) and
//       B (nb values b_j) and S sums with linear weights W[s][i][j]:
//         out_s = ha + hb + log2 sum_{i,j} W[s,i,j] 2^(a_i-ha) 2^(b_j-hb)
//       (exp distributes over the product node, so the max-shifted sum over
//       the na*nb products factorises).  Stage 1 on tcgen05:
//         T[m, (s,i)] = sum_j eb[m,j] W[s,i,j]   (M=128, K=nb, N=S*na groups)
//       with A = eb (f16, K-major in shared memory), B = the prepared weight
//       image, D accumulated in TMEM; stage 2 per sample on FP32:
//         out_s = ha + hb + lg2(sum_i ea[m,i] T[m,(s,i)])   (tcgen05.ld).
//       Precision: f16 operands, optionally split hi+lo (3 MMAs:
//       hi*hi + lo*hi + hi*lo, ~2^-22 relative) -- spn_prepare_options.tc_precision.
//  ROOT: the same contraction for the root region's partition of each
//       repetition, accumulated over repetitions by an online log-sum-exp;
//       the C class log-likelihoods and their argmax are written at the end.
#include <cuda_fp16.h>
#include <cuda_runtime.h>
#include <math_constants.h>
#include <stdint.h>
#include <stdlib.h>

#include "layered.h"

namespace spnb {



constexpr int RT = 128;   // samples per tile (= UMMA M, = TMEM lanes)
// threads per CTA: template parameter NTH of rat_eval_kernel (256 or 512)
constexpr uint32_t TMEM_BUF = 256;  // columns per accumulator buffer

__device__ __forceinline__ float r_ex2(float x) {
    float y;
    asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
    return y;
}
__device__ __forceinline__ float r_lg2(float x) {
    float y;
    asm("lg2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
    return y;
}
__device__ __forceinline__ float r_maxnan(float a, float b) {
    float r;
    asm("max.NaN.f32 %0, %1, %2;" : "=f"(r) : "f"(a), "f"(b));
    return r;
}
// log2(2^a + 2^b), NaN-propagating, -inf safe
__device__ __forceinline__ float r_lse2(float a, float b) {
    const float hi = r_maxnan(a, b), lo = fminf(a, b);
    return hi + r_lg2(1.f + r_ex2(lo - fmaxf(hi, -1e30f)));
}

__device__ __forceinline__ uint32_t r_smem(const void *p) {
    return (uint32_t)__cvta_generic_to_shared(p);
}

// UMMA shared-memory descriptor, K-major, no swizzle (canonical layout
// ((8,m),(T,2)):((16B,SBO),(1,LBO)); version 1 for sm_100).
__device__ __forceinline__ uint64_t umma_desc(uint32_t addr, uint32_t lbo, uint32_t sbo) {
    uint64_t d = 0;
    d |= (uint64_t)((addr >> 4) & 0x3FFFu);
    d |= (uint64_t)((lbo >> 4) & 0x3FFFu) << 16;
    d |= (uint64_t)((sbo >> 4) & 0x3FFFu) << 32;
    d |= (uint64_t)1 << 46;
    return d;
}

__device__ __forceinline__ void umma_f16(uint32_t d_tmem, uint64_t a, uint64_t b, uint32_t idesc,
                                         uint32_t accumulate) {
    asm volatile(
        "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}\n" ::"r"(d_tmem),
        "l"(a), "l"(b), "r"(idesc), "r"(accumulate));
}

__device__ __forceinline__ void umma_commit(uint32_t mbar) {
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(
                     mbar)
                 : "memory");
}

__device__ __forceinline__ void mbar_wait(uint32_t mbar, uint32_t parity) {
    uint32_t done = 0;
    while (!done) {
        asm volatile(
            "{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\t"
            "selp.u32 %0, 1, 0, p;\n\t}\n"
            : "=r"(done)
            : "r"(mbar), "r"(parity)
            : "memory");
    }
}

__device__ __forceinline__ void tmem_ld8(uint32_t taddr, float (&v)[8]) {
    uint32_t r[8];
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x8.b32 {%0, %1, %2, %3, %4, %5, %6, %7}, [%8];"
        : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]),
          "=r"(r[7])
        : "r"(taddr));
#pragma unroll
    for (int k = 0; k < 8; ++k) v[k] = __uint_as_float(r[k]);
}
__device__ __forceinline__ void tmem_ld4(uint32_t taddr, float (&v)[4]) {
    uint32_t r[4];
    asm volatile("tcgen05.ld.sync.aligned.32x32b.x4.b32 {%0, %1, %2, %3}, [%4];"
                 : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3])
                 : "r"(taddr));
#pragma unroll
    for (int k = 0; k < 4; ++k) v[k] = __uint_as_float(r[k]);
}
__device__ __forceinline__ void tmem_wait_ld() {
    asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
}
__device__ __forceinline__ void fence_before() {
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
}
__device__ __forceinline__ void fence_after() {
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
}
__device__ __forceinline__ void fence_async_smem() {
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}

// TMA bulk copy global -> shared, completion counted on an mbarrier (tx bytes)
__device__ __forceinline__ void bulk_g2s(uint32_t dst, const void *src, uint32_t bytes,
                                         uint32_t mbar) {
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
            dst),
        "l"(src), "r"(bytes), "r"(mbar)
        : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint32_t mbar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(mbar), "r"(bytes)
                 : "memory");
}

// element (row, k) of a K-major no-swizzle f16 operand image with `rows` rows
__device__ __forceinline__ uint32_t img_off(int row, int k, int rows) {
    return (uint32_t)((k >> 3) * (rows * 16) + (row >> 3) * 128 + (row & 7) * 16 + (k & 7) * 2);
}

// NaN-propagating max of V[i][m] over i < n: four independent chains (the
// loads of a chain issue back to back instead of one dependent max per load)
__device__ __forceinline__ float col_max(const float *V, int n, int m) {
    float h[4] = {-CUDART_INF_F, -CUDART_INF_F, -CUDART_INF_F, -CUDART_INF_F};
    int i = 0;
    for (; i + 4 <= n; i += 4) {
#pragma unroll
        for (int k = 0; k < 4; ++k) h[k] = r_maxnan(h[k], V[(i + k) * RT + m]);
    }
    for (; i < n; ++i) h[0] = r_maxnan(h[0], V[i * RT + m]);
    return r_maxnan(r_maxnan(h[0], h[1]), r_maxnan(h[2], h[3]));
}

// LEAF step: the region's feature rows xs[v][m] (128 samples) and its
// parameter block ab[v][i] = (a, b), C[i] are in shared memory (one bulk-copy
// stage).  256 threads = 32 sample quads x 8 distribution groups of DPT =
// I/8 distributions; per variable a thread does 1 LDS.128 (x) + DPT LDS.64
// (broadcast) for 8 DPT FFMA.
#ifndef LEAF_UNROLL
#define LEAF_UNROLL 8
#endif
constexpr int kLeafUnroll = LEAF_UNROLL;
#ifndef W_CHUNKS
#define W_CHUNKS 1  // concurrent bulk copies per weight-group part
#endif  // variable loop of a LEAF step
// 512-thread mapping: 64 sample pairs x 8 distribution groups of DPT; per
// variable 1 LDS.64 (x pair) + DPT LDS.64 (broadcast (a, b)) for 2 DPT FFMA2.
template <int DPT, bool MARG>
__device__ __forceinline__ void leaf_step_pairs(const LStep &st, float *act, const float *xs,
                                                const float *prm, int tid) {
    const int I = st.n_out, V = st.n_vars;
    const int mp = (tid & 63) * 2;           // 2 samples
    const int grp = tid >> 6, d0 = grp * DPT; // distribution group, first distribution
    constexpr int DPTP = DPT + (DPT & 1);    // pairs per (v, group), padded to even
    const float4 *ab4 = reinterpret_cast<const float4 *>(prm) + grp * (DPTP / 2);
    const float *C = prm + (st.cst_off - st.par_off);
    float2 acc[DPT];
#pragma unroll
    for (int d = 0; d < DPT; ++d) acc[d] = make_float2(C[d0 + d], C[d0 + d]);
    const float K0 = -1.0901312512f;  // 0.5 * log2(ln2 / pi)
#pragma unroll (kLeafUnroll)
    for (int v = 0; v < V; ++v) {
        const float2 x2 = *reinterpret_cast<const float2 *>(xs + v * RT + mp);
        bool anynan = false;
        if constexpr (MARG) anynan = (x2.x != x2.x) | (x2.y != x2.y);
        float2 qv[DPTP];
#pragma unroll
        for (int k = 0; k < DPTP / 2; ++k) {  // two (a, b) pairs per LDS.128
            const float4 q4 = ab4[v * 4 * DPTP + k];
            qv[2 * k] = make_float2(q4.x, q4.y);
            qv[2 * k + 1] = make_float2(q4.z, q4.w);
        }
#pragma unroll
        for (int d = 0; d < DPT; ++d) {
            const float2 q = qv[d];
            if (MARG && anynan) {
                const float cc = r_lg2(q.x) + K0;
                const float t0 = fmaf(q.x, x2.x, -q.y), t1 = fmaf(q.x, x2.y, -q.y);
                const bool n0 = x2.x != x2.x, n1 = x2.y != x2.y;
                acc[d].x = fmaf(-(n0 ? cc : t0), n0 ? 1.f : t0, acc[d].x);
                acc[d].y = fmaf(-(n1 ? cc : t1), n1 ? 1.f : t1, acc[d].y);
            } else {
                const float2 t = __ffma2_rn(x2, make_float2(q.x, q.x), make_float2(-q.y, -q.y));
                acc[d] = __ffma2_rn(make_float2(-t.x, -t.y), t, acc[d]);
            }
        }
    }
#pragma unroll
    for (int d = 0; d < DPT; ++d)
        *reinterpret_cast<float2 *>(act + st.buf_out + (d0 + d) * RT + mp) = acc[d];
}

template <int DPT, bool MARG, int NTH>
__device__ __forceinline__ void leaf_step_t(const LStep &st, float *act, const float *xs,
                                            const float *prm, int tid) {
    if constexpr (NTH == 512) {
        leaf_step_pairs<DPT, MARG>(st, act, xs, prm, tid);
        return;
    }
    const int I = st.n_out, V = st.n_vars;
    const int mq = (tid & 31) * 4;           // 4 samples
    const int grp = tid >> 5, d0 = grp * DPT; // distribution group, first distribution
    constexpr int DPTP = DPT + (DPT & 1);    // pairs per (v, group), padded to even
    const float4 *ab4 = reinterpret_cast<const float4 *>(prm) + grp * (DPTP / 2);
    const float *C = prm + (st.cst_off - st.par_off);
    float acc[DPT][4];
#pragma unroll
    for (int d = 0; d < DPT; ++d) {
        const float cd = C[d0 + d];
        acc[d][0] = cd; acc[d][1] = cd; acc[d][2] = cd; acc[d][3] = cd;
    }
    // log2 N = c - t^2 with c = log2(a) + K0 (used only to cancel a NaN leaf)
    const float K0 = -1.0901312512f;  // 0.5 * log2(ln2 / pi)
#pragma unroll (kLeafUnroll)
    for (int v = 0; v < V; ++v) {
        const float4 x4 = *reinterpret_cast<const float4 *>(xs + v * RT + mq);
        const float xv[4] = {x4.x, x4.y, x4.z, x4.w};
        bool anynan = false;
        if constexpr (MARG) anynan = (xv[0] != xv[0]) | (xv[1] != xv[1]) | (xv[2] != xv[2]) | (xv[3] != xv[3]);
        float2 qv[DPTP];
#pragma unroll
        for (int k = 0; k < DPTP / 2; ++k) {  // two (a, b) pairs per LDS.128
            const float4 q4 = ab4[v * 4 * DPTP + k];
            qv[2 * k] = make_float2(q4.x, q4.y);
            qv[2 * k + 1] = make_float2(q4.z, q4.w);
        }
#pragma unroll
        for (int d = 0; d < DPT; ++d) {
            const float2 q = qv[d];
            if (MARG && anynan) {
                const float cc = r_lg2(q.x) + K0;
#pragma unroll
                for (int k = 0; k < 4; ++k) {
                    const bool nan = xv[k] != xv[k];
                    const float t = fmaf(q.x, xv[k], -q.y);
                    acc[d][k] = fmaf(-(nan ? cc : t), nan ? 1.f : t, acc[d][k]);
                }
            } else {
                // packed FP32 (FFMA2, sm_100): two samples per instruction, the
                // parameters broadcast (.F32) and -b folded as an operand modifier
                const float2 a2 = make_float2(q.x, q.x), nb2 = make_float2(-q.y, -q.y);
                const float2 t01 = __ffma2_rn(make_float2(xv[0], xv[1]), a2, nb2);
                const float2 t23 = __ffma2_rn(make_float2(xv[2], xv[3]), a2, nb2);
                const float2 s01 = __ffma2_rn(make_float2(-t01.x, -t01.y), t01,
                                              make_float2(acc[d][0], acc[d][1]));
                const float2 s23 = __ffma2_rn(make_float2(-t23.x, -t23.y), t23,
                                              make_float2(acc[d][2], acc[d][3]));
                acc[d][0] = s01.x; acc[d][1] = s01.y; acc[d][2] = s23.x; acc[d][3] = s23.y;
            }
        }
    }
#pragma unroll
    for (int d = 0; d < DPT; ++d)
        *reinterpret_cast<float4 *>(act + st.buf_out + (d0 + d) * RT + mq) =
            make_float4(acc[d][0], acc[d][1], acc[d][2], acc[d][3]);
}

template <bool MARG, int NTH>
__device__ void leaf_step(const LStep &st, float *act, const float *xs, const float *prm, int tid) {
    switch (st.n_out >> 3) {
        case 1: leaf_step_t<1, MARG, NTH>(st, act, xs, prm, tid); break;
        case 2: leaf_step_t<2, MARG, NTH>(st, act, xs, prm, tid); break;
        case 3: leaf_step_t<3, MARG, NTH>(st, act, xs, prm, tid); break;
        case 4: leaf_step_t<4, MARG, NTH>(st, act, xs, prm, tid); break;
        case 5: leaf_step_t<5, MARG, NTH>(st, act, xs, prm, tid); break;
        case 6: leaf_step_t<6, MARG, NTH>(st, act, xs, prm, tid); break;
        case 7: leaf_step_t<7, MARG, NTH>(st, act, xs, prm, tid); break;
        case 8: leaf_step_t<8, MARG, NTH>(st, act, xs, prm, tid); break;
    }
}

template <bool MARG, int NTH>
__global__ void __launch_bounds__(NTH, 1) rat_eval_kernel(const RParams p) {
    constexpr int NSPLIT = NTH / RT;    // epilogue: warps per TMEM lane quarter
    constexpr int EA_MAX = NTH == 512 ? 48 : 64;  // ea values per thread in registers
#ifndef EPI_SPS
#define EPI_SPS 1
#endif
    constexpr int SPS = NTH == 512 ? 1 : EPI_SPS;  // sums per TMEM wait in the epilogue
    extern __shared__ __align__(1024) uint8_t smem[];
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    // samples: from the launch, or counted on the device (certification fallback)
    int64_t n = p.n;
    if (p.n_count) n = max((int64_t)0, min(n, (int64_t)*p.n_count - p.n_off));
    if (n <= 0) return;
    // ---- shared-memory carve-up (mirrored by rat_smem_bytes) ----
    uint64_t *bars = reinterpret_cast<uint64_t *>(smem);  // 0 mma, 1-3 w, 4/5 x
    uint32_t *tmem_slot = reinterpret_cast<uint32_t *>(smem + 64);
    size_t off = 128;
    float *act = reinterpret_cast<float *>(smem + off);
    off += (size_t)p.smem_floats * 4;
    float *racc = reinterpret_cast<float *>(smem + off);
    off += (size_t)p.C * RT * 4;
    float *ea = reinterpret_cast<float *>(smem + off);
    off += (size_t)p.max_na * RT * 4;
    float *sa = reinterpret_cast<float *>(smem + off);
    float *sb = sa + RT;
    off += 2 * RT * 4;
    // leaf staging, 2 buffers of [max_vars][RT] x rows + [max_leaf_params] params
    const size_t stage_floats = (size_t)p.max_vars * RT + (size_t)p.max_leaf_params;
    float *xsb = reinterpret_cast<float *>(smem + off);
    off += 2 * stage_floats * 4;
    off = (off + 1023) & ~(size_t)1023;
    uint8_t *aimg = smem + off;  // [2][RT x kpad] f16 (hi, lo)
    const size_t aimg_part = (size_t)RT * p.max_kpad * 2;
    off += 2 * aimg_part;
    off = (off + 1023) & ~(size_t)1023;
    uint8_t *wsm = smem + off;   // [wbufs][prec==3 ? 2 : 1][n_group x kpad] f16
    const size_t w_part = (size_t)p.max_ngroup * p.max_kpad * 2;
    const size_t w_buf = w_part * (p.prec == 3 ? 2 : 1);
    const bool ovl = p.wbufs >= 2 && p.overlap;
    const uint32_t tmem_cols = ovl ? 2 * TMEM_BUF : TMEM_BUF;

    const uint32_t bar_mma = r_smem(bars), bar_w0 = r_smem(bars + 1);
    const uint32_t bar_x0 = r_smem(bars + 4);
    if (warp == 0) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(
                         r_smem(tmem_slot)),
                     "r"(tmem_cols));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    if (tid == 0) {
        for (int i = 0; i < 6; ++i)
            asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(r_smem(bars + i)), "r"(1));
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    fence_before();
    __syncthreads();
    fence_after();
    const uint32_t tmem = *tmem_slot;
    uint32_t ph_mma = 0, ph_w = 0, ph_x = 0;  // phase parity bits (bit b: buffer b)
    int xbuf = 0;  // buffer of the next leaf step

    // x rows + parameter block of a leaf step for the tile at `base` -> buffer
    // b; issued by the lanes of warp 0 (one bulk copy per lane)
    auto issue_x = [&](int step, int64_t base, int b) {
        const LStep &ls = p.steps[step];
        const int nv = ls.n_vars;
        const uint32_t dst = r_smem(xsb + (size_t)b * stage_floats);
        const uint32_t bar = bar_x0 + 8 * b;
        const uint32_t pbytes = (uint32_t)ls.w_off * 4;
        if (lane == 0) {
            mbar_expect_tx(bar, (uint32_t)nv * RT * 4 + pbytes);
            bulk_g2s(dst + (uint32_t)p.max_vars * RT * 4, p.fparams + ls.par_off, pbytes, bar);
        }
        __syncwarp();
        for (int v = lane; v < nv; v += 32) {
            const int f = __ldg(p.vars + ls.vars_off + v);
            bulk_g2s(dst + v * RT * 4, p.xT + (int64_t)f * p.ldT + base, RT * 4, bar);
        }
    };
    // weight group g of step ws -> buffer b; issued by the lanes of warp 0 as
    // W_CHUNKS concurrent bulk copies per operand part (one large copy per
    // part measured slower: the copies of one SM are serviced in parallel)
    auto issue_w = [&](const LStep &ws, int g, int b) {
        const uint32_t gb = (uint32_t)ws.w_group_bytes;
        const uint8_t *src = p.wimg + ws.w_off + 2 * (size_t)gb * g;
        const uint32_t bar = bar_w0 + 8 * b;
        const uint32_t dst = r_smem(wsm) + (uint32_t)(b * w_buf);
        const int parts = p.prec == 3 ? 2 : 1;
        if (lane == 0) mbar_expect_tx(bar, gb * parts);
        __syncwarp();
        const uint32_t cb = ((gb + W_CHUNKS - 1) / W_CHUNKS + 15) & ~15u;  // 16-B multiple
        for (int k = lane; k < W_CHUNKS * parts; k += 32) {
            const int part = k / W_CHUNKS;
            const uint32_t o = (uint32_t)(k % W_CHUNKS) * cb;
            if (o < gb)
                bulk_g2s(dst + (uint32_t)part * (uint32_t)w_part + o, src + (size_t)part * gb + o,
                         min(cb, gb - o), bar);
        }
    };

    const int64_t n_tiles = (n + RT - 1) / RT;
    // optional profiling: cycles per phase measured by thread 0
    unsigned long long pc_acc[8] = {0, 0, 0, 0, 0, 0, 0, 0};
    unsigned long long t_mark = clock64();
    auto prof_mark = [&](int k) {
        if (p.prof && tid == 0) {
            const unsigned long long t = clock64();
            pc_acc[k] += t - t_mark;
            t_mark = t;
        }
    };
    if (warp == 0 && (int64_t)blockIdx.x < n_tiles) issue_x(p.first_leaf, (int64_t)blockIdx.x * RT, 0);
    for (int64_t tile = blockIdx.x; tile < n_tiles; tile += gridDim.x) {
        const int64_t base = tile * RT;
        for (int i = tid; i < p.C * RT; i += NTH) racc[i] = -CUDART_INF_F;
        __syncthreads();
        for (int si = 0; si < p.n_steps; ++si) {
            const LStep st = p.steps[si];  // by value: fields live in registers
            if (st.type == 0) {
                const int b = xbuf;
                prof_mark(7);
                mbar_wait(bar_x0 + 8 * b, (ph_x >> b) & 1u);
                ph_x ^= 1u << b;
                prof_mark(0);  // 0: waiting for the leaf rows
                if (warp == 0) {  // prefetch the next leaf step's rows (maybe next tile)
                    if (st.rep >= 0) issue_x(st.rep, base, b ^ 1);
                    else if (tile + gridDim.x < n_tiles)
                        issue_x(p.first_leaf, base + (int64_t)gridDim.x * RT, b ^ 1);
                }
                xbuf ^= 1;
                {
                    const float *stg = xsb + (size_t)b * stage_floats;
                    leaf_step<MARG, NTH>(st, act, stg, stg + (size_t)p.max_vars * RT, tid);
                }
                prof_mark(1);  // 1: leaf compute
                __syncthreads();
                prof_mark(2);  // 2: leaf barrier
                continue;
            }
            // ---------------- SUM / ROOT: phase 1 (shifts, exps, A image) ----
            const int G = st.n_groups;
            if (warp == 0) {
                for (int b = 0; b < p.wbufs && b < G; ++b) issue_w(st, b, b);
            }
            const int na = st.na, nb = st.nb, kpad = st.k_pad;
            // NTH/2 threads per side: PH = NTH/256 threads per sample (warps
            // w and w+4 share a sample), each computes the full max and
            // 1/PH of the exps (no extra barrier to combine maxima)
            constexpr int PH = NTH / 256;
            const int side = tid / (NTH / 2), ts = tid % (NTH / 2);
            const int m = ((ts >> 5) & 3) * 32 + lane, ph = ts >> 7;
            if (side == 0) {
                const float *VA = act + st.buf_a;
                const float hi = col_max(VA, na, m);
                const float hc = fmaxf(hi, -1e30f);
                const int ic = (na + PH - 1) / PH;
                for (int i = ph * ic; i < min(na, (ph + 1) * ic); ++i)
                    ea[i * RT + m] = r_ex2(VA[i * RT + m] - hc);
                if (ph == 0) sa[m] = hi;
            } else {
                const float *VB = act + st.buf_b;
                const float hi = col_max(VB, nb, m);
                const float hc = fmaxf(hi, -1e30f);
                for (int j0 = ph * 8; j0 < kpad; j0 += 8 * PH) {  // 8 k-values = one 16-byte row
                    uint32_t hw[4], lw[4];
#pragma unroll
                    for (int k = 0; k < 8; k += 2) {
                        const int j = j0 + k;
                        const float e0 = j < nb ? r_ex2(VB[j * RT + m] - hc) : 0.f;
                        const float e1 = j + 1 < nb ? r_ex2(VB[(j + 1) * RT + m] - hc) : 0.f;
                        const __half h0 = __float2half_rn(e0), h1 = __float2half_rn(e1);
                        const __half l0 = __float2half_rn(e0 - __half2float(h0));
                        const __half l1 = __float2half_rn(e1 - __half2float(h1));
                        hw[k >> 1] = (uint32_t)__half_as_ushort(h0) | ((uint32_t)__half_as_ushort(h1) << 16);
                        lw[k >> 1] = (uint32_t)__half_as_ushort(l0) | ((uint32_t)__half_as_ushort(l1) << 16);
                    }
                    const uint32_t o = img_off(m, j0, RT);
                    *reinterpret_cast<uint4 *>(aimg + o) = make_uint4(hw[0], hw[1], hw[2], hw[3]);
                    *reinterpret_cast<uint4 *>(aimg + aimg_part + o) = make_uint4(lw[0], lw[1], lw[2], lw[3]);
                }
                if (ph == 0) sb[m] = hi;
            }
            fence_async_smem();
            __syncthreads();
            prof_mark(3);  // 3: sum phase 1 (+barrier)
            // ---------------- phase 2: per N-group MMA + epilogue -------------
            const uint32_t lbo_a = RT * 16;
            const uint32_t lbo_b = (uint32_t)st.n_group * 16;
            const uint32_t idesc = (1u << 4) | ((uint32_t)(st.n_group >> 3) << 17) |
                                   ((uint32_t)(RT >> 4) << 24);
            const uint32_t a_hi = r_smem(aimg), a_lo = a_hi + (uint32_t)aimg_part;
            // epilogue of group g from TMEM buffer tb: warp quarter q reads
            // lanes 32q..32q+31 (= samples); the two warp halves split the sums
            // this thread's sample (TMEM lane quarter) and its ea values in
            // registers, reused by every sum of every group of this step
            const int qd = warp & 3, part = warp >> 2;
            const int m_ep = qd * 32 + lane;
            float ear[EA_MAX];
#pragma unroll
            for (int i = 0; i < EA_MAX; ++i) ear[i] = i < na ? ea[i * RT + m_ep] : 0.f;
            const float shift = sa[m_ep] + sb[m_ep];
            auto epilogue = [&](int g, uint32_t tb) {
                const int m = m_ep;
                const int s0 = g * st.s_per_group;
                const int ns = min(st.s_per_group, st.n_out - s0);
                // the NSPLIT warps of a lane quarter split the group's sums
                const int sl0 = (ns * part) / NSPLIT, sl1 = (ns * (part + 1)) / NSPLIT;
                // SPS sums per TMEM wait: every column of those sums is loaded
                // (tcgen05.ld.32x32b, x8 / x4) before one tcgen05.wait::ld --
                // the wait covers all outstanding loads, so fewer, larger
                // batches mean fewer exposed TMEM latencies
                for (int sl = sl0; sl < sl1; sl += SPS) {
                    float t[SPS][EA_MAX];
#pragma unroll
                    for (int u = 0; u < SPS; ++u) {
                        const bool live = sl + u < sl1;
                        const uint32_t trow = tmem + tb + ((uint32_t)(qd * 32) << 16) +
                                              (uint32_t)((sl + u) * na);
#pragma unroll
                        for (int c0 = 0; c0 < EA_MAX; c0 += 8) {
                            if (live && c0 + 8 <= na) {
                                float v8[8];
                                tmem_ld8(trow + c0, v8);
#pragma unroll
                                for (int k = 0; k < 8; ++k) t[u][c0 + k] = v8[k];
                            } else if (live && c0 < na) {
                                float v4[4];
                                tmem_ld4(trow + c0, v4);
#pragma unroll
                                for (int k = 0; k < 4; ++k) {
                                    t[u][c0 + k] = v4[k];
                                    t[u][c0 + 4 + k] = 0.f;
                                }
                            } else {
#pragma unroll
                                for (int k = 0; k < 8; ++k) t[u][c0 + k] = 0.f;
                            }
                        }
                    }
                    tmem_wait_ld();
#pragma unroll
                    for (int u = 0; u < SPS; ++u) {
                        if (sl + u >= sl1) break;
                        // packed FP32 (FFMA2): 2 x 2 independent chains
                        float2 p01 = make_float2(0.f, 0.f), p23 = make_float2(0.f, 0.f);
#pragma unroll
                        for (int i = 0; i < EA_MAX; i += 4) {
                            p01 = __ffma2_rn(make_float2(ear[i], ear[i + 1]),
                                             make_float2(t[u][i], t[u][i + 1]), p01);
                            p23 = __ffma2_rn(make_float2(ear[i + 2], ear[i + 3]),
                                             make_float2(t[u][i + 2], t[u][i + 3]), p23);
                        }
                        const float acc = (p01.x + p01.y) + (p23.x + p23.y);
                        const float val = shift + r_lg2(acc);
                        const int s = s0 + sl + u;
                        if (st.type == 1) {
                            act[st.buf_out + s * RT + m] = val;
                        } else {
                            const int col = __ldg(p.root_map + s);
                            racc[col * RT + m] = r_lse2(racc[col * RT + m], val);
                        }
                    }
                }
            };
            for (int g = 0; g < G; ++g) {
                const int wb = g % p.wbufs;  // ring of wbufs weight buffers
                const uint32_t tb = ovl ? (uint32_t)(g & 1) * TMEM_BUF : 0u;
                mbar_wait(bar_w0 + 8 * wb, (ph_w >> wb) & 1u);
                ph_w ^= 1u << wb;
                prof_mark(4);  // 4: waiting for weights
                if (tid == 0) {
                    fence_after();
                    const uint32_t w_hi = r_smem(wsm) + (uint32_t)(wb * w_buf);
                    const uint32_t w_lo = w_hi + (uint32_t)w_part;
                    for (int kk = 0; kk < kpad / 16; ++kk) {
                        const uint32_t ka = kk * 2 * lbo_a, kb = kk * 2 * lbo_b;
                        umma_f16(tmem + tb, umma_desc(a_hi + ka, lbo_a, 128),
                                 umma_desc(w_hi + kb, lbo_b, 128), idesc, kk > 0);
                        if (p.prec == 3) {
                            umma_f16(tmem + tb, umma_desc(a_lo + ka, lbo_a, 128),
                                     umma_desc(w_hi + kb, lbo_b, 128), idesc, 1);
                            umma_f16(tmem + tb, umma_desc(a_hi + ka, lbo_a, 128),
                                     umma_desc(w_lo + kb, lbo_b, 128), idesc, 1);
                        }
                    }
                    umma_commit(bar_mma);
                }
                __syncwarp();
                // overlap: the previous group's epilogue runs under this MMA
                if (ovl && g > 0) epilogue(g - 1, (uint32_t)((g - 1) & 1) * TMEM_BUF);
                prof_mark(5);  // 5: MMA issue + overlapped epilogue
                mbar_wait(bar_mma, ph_mma);
                ph_mma ^= 1;
                fence_after();
                prof_mark(6);  // 6: waiting for the MMA
                // the MMA has consumed weight buffer wb: refill it
                if (warp == 0 && g + p.wbufs < G) issue_w(st, g + p.wbufs, wb);
                if (!ovl) epilogue(g, 0u);
                fence_before();
                __syncthreads();
            }
            if (ovl) {
                epilogue(G - 1, (uint32_t)((G - 1) & 1) * TMEM_BUF);
                fence_before();
                __syncthreads();
            }
        }
        // ---------------- outputs -------------------------------------------
        if (tid < RT) {
            const int64_t srow = base + tid;
            if (srow < n) {
                int best = -1;
                float bv = -CUDART_INF_F;
                for (int c = 0; c < p.C; ++c) {
                    const float v = racc[c * RT + tid] * 0.6931471805599453f;
                    p.out[srow * p.C + c] = v;
                    if (!(v != v) && (best < 0 || v > bv)) {
                        best = c;
                        bv = v;
                    }
                }
                if (p.argmax) p.argmax[srow] = best;
            }
        }
        __syncthreads();
    }
    if (p.prof && tid == 0)
        for (int k = 0; k < 8; ++k) atomicAdd(p.prof + k, pc_acc[k]);
    fence_before();
    __syncthreads();
    if (warp == 0)
        asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem),
                     "r"(tmem_cols));
}

// xT[f][s] = x[s][f] for s < n (zero for n <= s < rows_pad)
__global__ void transpose_x_kernel(const float *__restrict__ x, int64_t n, int64_t ld, int F,
                                   float *__restrict__ xT, int64_t ldT, int64_t rows_pad) {
    __shared__ float t[32][33];
    // row blocks on grid.x (up to 2^31-1), feature blocks on grid.y
    const int64_t s0 = (int64_t)blockIdx.x * 32, f0 = (int64_t)blockIdx.y * 32;
    const int tx = threadIdx.x, ty = threadIdx.y;  // 32 x 8
    for (int k = ty; k < 32; k += 8) {
        const int64_t s = s0 + k, f = f0 + tx;
        t[k][tx] = (s < n && f < F) ? __ldg(x + s * ld + f) : 0.f;
    }
    __syncthreads();
    for (int k = ty; k < 32; k += 8) {
        const int64_t f = f0 + k, s = s0 + tx;
        if (f < F && s < rows_pad) xT[f * ldT + s] = t[tx][k];
    }
}

// certification fallback: xT[f][k] = x[idx[off + k]][f] for the flagged rows
// k < min(*count - off, cap) (zero for the rest of each 32-row block)
__global__ void gather_transpose_kernel(const float *__restrict__ x, int64_t ld, int F,
                                        const int64_t *__restrict__ idx, const int32_t *count,
                                        int64_t off, int64_t cap, float *__restrict__ xT,
                                        int64_t ldT) {
    const int64_t m = max((int64_t)0, min(cap, (int64_t)*count - off));
    const int64_t s0 = (int64_t)blockIdx.x * 32, f0 = (int64_t)blockIdx.y * 32;
    if (s0 >= m) return;
    __shared__ float t[32][33];
    const int tx = threadIdx.x, ty = threadIdx.y;
    for (int k = ty; k < 32; k += 8) {
        const int64_t s = s0 + k, f = f0 + tx;
        t[k][tx] = (s < m && f < F) ? __ldg(x + __ldg(idx + off + s) * ld + f) : 0.f;
    }
    __syncthreads();
    for (int k = ty; k < 32; k += 8) {
        const int64_t f = f0 + k, s = s0 + tx;
        if (f < F) xT[f * ldT + s] = t[tx][k];
    }
}

// certification fallback: out[idx[off + k]] = tmp[k] (and argmax) for the flagged rows
__global__ void scatter_rows_kernel(const float *__restrict__ tmp, const int32_t *__restrict__ am_tmp,
                                    const int64_t *__restrict__ idx, const int32_t *count,
                                    int64_t off, int64_t cap, int C, float *__restrict__ out,
                                    int32_t *__restrict__ am) {
    const int64_t m = max((int64_t)0, min(cap, (int64_t)*count - off));
    for (int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; k < m;
         k += (int64_t)gridDim.x * blockDim.x) {
        const int64_t r = __ldg(idx + off + k);
        for (int c = 0; c < C; ++c) out[r * C + c] = tmp[k * C + c];
        if (am) am[r] = am_tmp[k];
    }
}

cudaError_t cert_gather_launch(const float *x, int64_t ld, int F, const int64_t *idx,
                               const int32_t *count, int64_t off, int64_t cap, float *xT,
                               int64_t ldT, cudaStream_t st) {
    dim3 grid((unsigned)((cap + 31) / 32), (unsigned)((F + 31) / 32));
    gather_transpose_kernel<<<grid, dim3(32, 8), 0, st>>>(x, ld, F, idx, count, off, cap, xT, ldT);
    return cudaGetLastError();
}

cudaError_t cert_scatter_launch(const float *tmp, const int32_t *am_tmp, const int64_t *idx,
                                const int32_t *count, int64_t off, int64_t cap, int C, float *out,
                                int32_t *am, cudaStream_t st) {
    scatter_rows_kernel<<<148, 256, 0, st>>>(tmp, am_tmp, idx, count, off, cap, C, out, am);
    return cudaGetLastError();
}

size_t rat_smem_bytes(int smem_floats, int C, int max_na, int max_kpad, int max_ngroup,
                      int max_vars, int max_leaf_params, int prec, int wbufs) {
    size_t off = 128 + (size_t)smem_floats * 4 + (size_t)C * RT * 4 + (size_t)max_na * RT * 4 +
                 2 * RT * 4 + 2 * ((size_t)max_vars * RT + (size_t)max_leaf_params) * 4;
    off = (off + 1023) & ~(size_t)1023;
    off += 2 * (size_t)RT * max_kpad * 2;
    off = (off + 1023) & ~(size_t)1023;
    off += (size_t)wbufs * (prec == 3 ? 2 : 1) * (size_t)max_ngroup * max_kpad * 2;
    return off + 1024;  // alignment slack for the dynamic base
}

cudaError_t rat_launch(const RParams &p, bool marg, int grid, size_t smem, cudaStream_t st) {
    // 512 threads (16 warps) when the ea rows fit the 48-register epilogue
    // array, else 256; SPNB_RAT_THREADS=256 pins the 8-warp variant (A/B)
    static const int pin = [] {
        const char *e = getenv("SPNB_RAT_THREADS");
        return e ? atoi(e) : 0;
    }();
    const int nth = (pin == 256 || p.max_na > 48) ? 256 : 512;
    auto fn = nth == 512 ? (marg ? rat_eval_kernel<true, 512> : rat_eval_kernel<false, 512>)
                         : (marg ? rat_eval_kernel<true, 256> : rat_eval_kernel<false, 256>);
    cudaError_t e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    fn<<<grid, nth, smem, st>>>(p);
    return cudaGetLastError();
}

cudaError_t transpose_launch(const float *x, int64_t n, int64_t ld, int F, float *xT, int64_t ldT,
                             int64_t rows_pad, cudaStream_t st) {
    dim3 grid((unsigned)((rows_pad + 31) / 32), (unsigned)((F + 31) / 32));
    transpose_x_kernel<<<grid, dim3(32, 8), 0, st>>>(x, n, ld, F, xT, ldT, rows_pad);
    return cudaGetLastError();
}

}  // namespace spnb
