// api.cpp -- the C ABI of libspnb (include/spnb.h): handles, validation,
// plan preparation (launch-configuration choice + device upload), inference
// launches and the host-buffer end-to-end pipeline.
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

#include <algorithm>
#include <chrono>
#include <cmath>
#include <atomic>
#include <mutex>
#include <thread>
#include <new>
#include <string>
#include <vector>

#include "codegen.h"
#include "jit.h"
#include "layered.h"
#include "prepare.h"
#include "program.h"
#include "spnb.h"

namespace spnb {
cudaError_t dag_eval_launch_k1(const KParams &, bool, bool, int, int, size_t, cudaStream_t);
cudaError_t dag_eval_launch_k2(const KParams &, bool, bool, int, int, size_t, cudaStream_t);
cudaError_t dag_eval_launch_k4(const KParams &, bool, bool, int, int, size_t, cudaStream_t);
cudaError_t dag_eval_launch_k8(const KParams &, bool, bool, int, int, size_t, cudaStream_t);
int dag_eval_occupancy_k8(bool, bool, int, size_t);
int dag_eval_occupancy_k1(bool, bool, int, size_t);
int dag_eval_occupancy_k2(bool, bool, int, size_t);
int dag_eval_occupancy_k4(bool, bool, int, size_t);
// RParams: layered.h

size_t rat_smem_bytes(int smem_floats, int C, int max_na, int max_kpad, int max_ngroup,
                      int max_vars, int max_leaf_params, int prec, int wbufs);
cudaError_t rat_launch(const RParams &p, bool marg, int grid, size_t smem, cudaStream_t st);
cudaError_t transpose_launch(const float *x, int64_t n, int64_t ld, int F, float *xT, int64_t ldT,
                             int64_t rows_pad, cudaStream_t st);
bool rat2_supported_shape(int I, int S);
int rat2_layout(R2Params &p, int I, int max_vars, int max_blk, int kpad_bot, int kpad_up,
                int max_wgroup, int prec, int n_in, int n_w, int lvp, int kl_j, int kl_m);
cudaError_t cert_gather_launch(const float *x, int64_t ld, int F, const int64_t *idx,
                               const int32_t *count, int64_t off, int64_t cap, float *xT,
                               int64_t ldT, cudaStream_t st);
cudaError_t cert_scatter_launch(const float *tmp, const int32_t *am_tmp, const int64_t *idx,
                                const int32_t *count, int64_t off, int64_t cap, int C, float *out,
                                int32_t *am, cudaStream_t st);
cudaError_t rat2_launch(const R2Params &p, const int32_t *leaf_steps, int n_leaf,
                        const int32_t *sum_steps, int n_sum, bool marg, int grid, cudaStream_t st);
cudaError_t argmax_rows_launch(const float *out, int64_t n, int R, int32_t *argmax, cudaStream_t st);
}  // namespace spnb

using namespace spnb;

namespace {

thread_local std::string t_err;

int set_err(int code, const std::string &m) {
    t_err = m;
    return code;
}
int cuda_err(cudaError_t e, const char *where) {
    return set_err(SPN_E_CUDA, std::string(where) + ": " + cudaGetErrorString(e));
}

enum { H_GRAPH = 0x47524150, H_PLAN = 0x504c414e };

struct DevicePlan {
    int device = 0;
    int K = 4;
    bool xs = true;
    int tpw = 132;
    int block = 384;
    int grid_max = 0;        // persistent grid upper bound (SMs x CTAs/SM)
    int sms = 0;
    size_t smem = 0;
    int prog_cap = 0;
    int32_t F = 0, R = 0;
    int32_t n_tasks = 1;
    int32_t first_task_len = 0;
    int64_t n_sslots = 0, n_gslots = 0;
    Rec *d_prog = nullptr;
    int64_t *d_task_off = nullptr;
    float *d_tables = nullptr;
    Edge *d_edges = nullptr;
    float *d_gslots = nullptr;
    // plan-owned scratch (transposed features, interpreter global slots) is
    // used by one launch at a time: a call on a different stream than the
    // previous one waits for the previous one's event (spnb.h: re-entrant
    // across streams)
    std::mutex scratch_mu;
    cudaEvent_t scratch_ev = nullptr;
    void *scratch_stream = nullptr;
    // host pipeline buffers (lazily allocated)
    std::mutex host_mu;
    cudaStream_t hs[2] = {nullptr, nullptr};
    float *hx[2] = {nullptr, nullptr};
    float *hout[2] = {nullptr, nullptr};
    int32_t *ham[2] = {nullptr, nullptr};
    int64_t host_chunk = 0;
    // certified layered plans: whole groups of host rows resident on the
    // device (one certification round per group instead of one per chunk)
    float *gx = nullptr, *gout = nullptr;
    int32_t *gam = nullptr;
    int64_t group_cap = 0, group_piece = 0;
    std::vector<cudaEvent_t> gev;  // per piece (group_piece rows): its rows have landed
    cudaEvent_t gdone = nullptr;   // the group's kernels no longer read gx
    // layered (RAT-SPN) path
    int path = 0;
    LStep *d_steps = nullptr;
    int32_t n_steps = 0;
    int32_t *d_vars = nullptr;
    float *d_fparams = nullptr;
    uint8_t *d_wimg = nullptr;
    int32_t *d_root_map = nullptr;
    float *d_xT = nullptr;
    int64_t chunk = 0;
    int32_t prec = 3;
    int32_t smem_floats = 0, max_kpad = 0, max_ngroup = 0, max_na = 0;
    int32_t max_vars = 0, first_leaf = 0, max_leaf_params = 0, wbufs = 1;
    int32_t tmem_overlap = 1;  // epilogue of group g-1 under MMA g (SPNB_TMEM_OVERLAP=0: serial, A/B)
    unsigned long long *d_prof = nullptr;  // SPNB_PROFILE=1: phase cycle counters
    // layered v2: warp-specialised kernel (rat2.cu); used when the region
    // graph fits its constraints (build_rat2), else the v1 kernel above
    bool r2 = false;
    R2Params r2p;                 // device pointers + shared-memory layout
    R2Step *d_r2steps = nullptr;
    int32_t *d_r2vars = nullptr, *d_r2rm = nullptr, *d_r2leaf = nullptr, *d_r2sum = nullptr;
    float *d_r2fp = nullptr;
    uint8_t *d_r2w = nullptr;
    int32_t n_r2leaf = 0, n_r2sum = 0;
    // certified single pass (tc_precision auto): samples whose a-priori
    // error bound does not fit the tolerance are recomputed by v1 in hi/lo
    bool cert = false;
    bool leaf_tc = false;  // v2 with the leaf layer on the tensor cores
    float cert_err = 0.f;
    int32_t *d_flag_count = nullptr;
    int64_t *d_flag_idx = nullptr;  // grown (stream-ordered) to the largest n seen
    int64_t flag_cap = 0;
    float *d_cert_out = nullptr;
    int32_t *d_cert_am = nullptr;
    // compiled (per-SPN generated kernel) path
    std::vector<JitKernel> jk;
    std::vector<int32_t> jgrid_max;         // per task: SMs x CTAs/SM (joint kernel)
    std::vector<int32_t> jgrid_max_m;       // per task: SMs x CTAs/SM (marginal kernel)
    int jblock = 256;
    int jK = 1;  // samples per thread of the generated kernels
    bool jfused_argmax = false;
    float *d_jtab = nullptr;
    spn_plan_stats stats;
};

}  // namespace

struct spn_handle {
    uint32_t magic;
    GraphData *graph = nullptr;
    DevicePlan *plan = nullptr;
};

namespace {

int launch_kernel(const KParams &p, int K, bool marg, bool xs, int grid, int block, size_t smem,
                  cudaStream_t st) {
    cudaError_t e;
    switch (K) {
        case 8: e = dag_eval_launch_k8(p, marg, xs, grid, block, smem, st); break;
        case 4: e = dag_eval_launch_k4(p, marg, xs, grid, block, smem, st); break;
        case 2: e = dag_eval_launch_k2(p, marg, xs, grid, block, smem, st); break;
        case 1: e = dag_eval_launch_k1(p, marg, xs, grid, block, smem, st); break;
        default: return set_err(SPN_E_ARG, "bad samples_per_thread");
    }
    if (e != cudaSuccess) return cuda_err(e, "dag_eval launch");
    return SPN_OK;
}

int occupancy(int K, bool marg, bool xs, int block, size_t smem) {
    switch (K) {
        case 8: return dag_eval_occupancy_k8(marg, xs, block, smem);
        case 4: return dag_eval_occupancy_k4(marg, xs, block, smem);
        case 2: return dag_eval_occupancy_k2(marg, xs, block, smem);
        case 1: return dag_eval_occupancy_k1(marg, xs, block, smem);
    }
    return 0;
}

void free_plan(DevicePlan *p) {
    if (!p) return;
    int prev = -1;
    cudaGetDevice(&prev);
    cudaSetDevice(p->device);
    cudaFree(p->d_prog);
    cudaFree(p->d_task_off);
    cudaFree(p->d_tables);
    cudaFree(p->d_edges);
    cudaFree(p->d_gslots);
    cudaFree(p->d_steps);
    cudaFree(p->d_vars);
    cudaFree(p->d_fparams);
    cudaFree(p->d_wimg);
    cudaFree(p->d_root_map);
    cudaFree(p->d_xT);
    cudaFree(p->d_jtab);
    if (p->scratch_ev) cudaEventDestroy(p->scratch_ev);
    cudaFree(p->d_r2steps);
    cudaFree(p->d_r2vars);
    cudaFree(p->d_r2rm);
    cudaFree(p->d_r2leaf);
    cudaFree(p->d_r2sum);
    cudaFree(p->d_r2fp);
    cudaFree(p->d_r2w);
    cudaFree(p->d_flag_count);
    if (p->d_flag_idx) cudaFreeAsync(p->d_flag_idx, 0);
    cudaFree(p->d_cert_out);
    cudaFree(p->d_cert_am);
    for (auto &k : p->jk) jit_unload(k);
    if (p->d_prof) {
        unsigned long long h[8];
        if (!p->r2 && cudaMemcpy(h, p->d_prof, sizeof(h), cudaMemcpyDeviceToHost) == cudaSuccess) {
            const char *names[8] = {"leaf_wait", "leaf_compute", "leaf_barrier", "sum_phase1",
                                    "w_wait", "mma_issue+epilogue", "mma_wait", "other"};
            fprintf(stderr, "[spnb profile] cycles summed over CTAs:");
            for (int k = 0; k < 8; ++k) fprintf(stderr, " %s=%llu", names[k], h[k]);
            fprintf(stderr, "\n");
        }
        if (p->r2) {
            unsigned long long h2[32];
            if (cudaMemcpy(h2, p->d_prof, sizeof(h2), cudaMemcpyDeviceToHost) == cudaSuccess) {
                const char *roles[4] = {"leaf warps", "epilogue(8)", "mma", "producers"};
                const char *ph[4][8] = {
                    {"wait_in", "compute", "shift", "wait_out", "exp+write", "-", "-", "-"},
                    {"wait_leaf", "up_phase1", "wait_mma", "sums", "tile_io", "step_end", "ld_issue", "ld_wait"},
                    {"wait_A", "wait_w", "wait_tmem", "issue", "-", "-", "-", "-"},
                    {"wait_in_slot", "-", "wait_w_slot", "-", "-", "-", "-", "issue"}};
                for (int r = 0; r < 4; ++r) {
                    unsigned long long tot = 0;
                    for (int k = 0; k < 8; ++k) tot += h2[r * 8 + k];
                    fprintf(stderr, "[spnb profile v2] %-14s", roles[r]);
                    for (int k = 0; k < 8; ++k)
                        if (h2[r * 8 + k])
                            fprintf(stderr, " %s=%.1f%%", ph[r][k], 100.0 * h2[r * 8 + k] / (double)tot);
                    fprintf(stderr, "\n");
                }
            }
        }
        cudaFree(p->d_prof);
    }
    for (int i = 0; i < 2; ++i) {
        if (p->hs[i]) cudaStreamDestroy(p->hs[i]);
        cudaFree(p->hx[i]);
        if (i == 0) {
            cudaFree(p->gx);
            cudaFree(p->gout);
            cudaFree(p->gam);
            for (cudaEvent_t ev : p->gev) cudaEventDestroy(ev);
            if (p->gdone) cudaEventDestroy(p->gdone);
        }
        cudaFree(p->hout[i]);
        cudaFree(p->ham[i]);
    }
    if (prev >= 0) cudaSetDevice(prev);
    delete p;
}

struct DeviceGuard {
    int prev = -1;
    explicit DeviceGuard(int dev) {
        cudaGetDevice(&prev);
        if (prev != dev) cudaSetDevice(dev);
    }
    ~DeviceGuard() {
        int cur = -1;
        cudaGetDevice(&cur);
        if (prev >= 0 && cur != prev) cudaSetDevice(prev);
    }
};

template <typename T>
int upload(T **dst, const std::vector<T> &v) {
    const size_t bytes = std::max<size_t>(v.size(), 1) * sizeof(T);
    cudaError_t e = cudaMalloc((void **)dst, bytes);
    if (e != cudaSuccess) return e == cudaErrorMemoryAllocation ? set_err(SPN_E_OOM, "cudaMalloc")
                                                                 : cuda_err(e, "cudaMalloc");
    if (!v.empty()) {
        e = cudaMemcpy(*dst, v.data(), v.size() * sizeof(T), cudaMemcpyHostToDevice);
        if (e != cudaSuccess) return cuda_err(e, "cudaMemcpy");
    }
    return SPN_OK;
}

int infer_device_impl(spn_handle *h, const float *x, int64_t n, int64_t ld, float *out,
                      int32_t *argmax, void *stream, bool marg,
                      const cudaEvent_t *ready = nullptr, int64_t lchunk = 0);

int infer_device(spn_handle *h, const float *x, int64_t n, int64_t ld, float *out,
                 int32_t *argmax, void *stream, bool marg) {
    if (!h || h->magic != H_PLAN) return set_err(SPN_E_ARG, "not a plan handle");
    DevicePlan &P = *h->plan;
    const bool scratch = P.path == 1 || (P.path == 0 && P.n_gslots > 0);
    if (!scratch || n <= 0) return infer_device_impl(h, x, n, ld, out, argmax, stream, marg);
    std::lock_guard<std::mutex> lk(P.scratch_mu);
    DeviceGuard dg(P.device);
    cudaError_t e;
    if (P.scratch_ev && P.scratch_stream != stream &&
        (e = cudaStreamWaitEvent((cudaStream_t)stream, P.scratch_ev, 0)) != cudaSuccess)
        return cuda_err(e, "cudaStreamWaitEvent");
    const int rc = infer_device_impl(h, x, n, ld, out, argmax, stream, marg);
    if (rc != SPN_OK) return rc;
    if (!P.scratch_ev &&
        (e = cudaEventCreateWithFlags(&P.scratch_ev, cudaEventDisableTiming)) != cudaSuccess)
        return cuda_err(e, "cudaEventCreate");
    if ((e = cudaEventRecord(P.scratch_ev, (cudaStream_t)stream)) != cudaSuccess)
        return cuda_err(e, "cudaEventRecord");
    P.scratch_stream = stream;
    return SPN_OK;
}

// parameters of the v1 layered kernel (rat_eval.cu) of a plan
RParams v1_params(const DevicePlan &P) {
    RParams rp;
    memset(&rp, 0, sizeof(rp));
    rp.steps = P.d_steps;
    rp.n_steps = P.n_steps;
    rp.C = P.R;
    rp.vars = P.d_vars;
    rp.fparams = P.d_fparams;
    rp.wimg = P.d_wimg;
    rp.root_map = P.d_root_map;
    rp.prec = P.prec;
    rp.smem_floats = P.smem_floats;
    rp.max_kpad = P.max_kpad;
    rp.max_ngroup = P.max_ngroup;
    rp.max_na = P.max_na;
    rp.max_vars = P.max_vars;
    rp.first_leaf = P.first_leaf;
    rp.max_leaf_params = P.max_leaf_params;
    rp.wbufs = P.wbufs;
    rp.overlap = P.tmem_overlap;
    rp.prof = P.r2 ? nullptr : P.d_prof;
    return rp;
}

int infer_device_impl(spn_handle *h, const float *x, int64_t n, int64_t ld, float *out,
                      int32_t *argmax, void *stream, bool marg,
                      const cudaEvent_t *ready, int64_t lchunk) {
    if (!h || h->magic != H_PLAN) return set_err(SPN_E_ARG, "not a plan handle");
    DevicePlan &P = *h->plan;
    if (n < 0) return set_err(SPN_E_ARG, "n < 0");
    if (n == 0) return SPN_OK;
    if (!x || !out) return set_err(SPN_E_ARG, "null x/out");
    if (ld < P.F) return set_err(SPN_E_ARG, "ld < n_features");
    DeviceGuard dg(P.device);
    if (P.path == 2) {
        std::string msg;
        const int32_t *tasks_am = P.jfused_argmax ? argmax : nullptr;
        for (size_t t = 0; t < P.jk.size(); ++t) {
            const int64_t blk = P.jk[t].block[marg ? 1 : 0];
            const int64_t need = (n + blk * P.jK - 1) / (blk * P.jK);
            const int grid = (int)std::max<int64_t>(
                1, std::min<int64_t>(need, marg ? P.jgrid_max_m[t] : P.jgrid_max[t]));
            const int rc = jit_launch(P.jk[t], marg, grid, (int)blk, (cudaStream_t)stream, x, n, ld,
                                      out, P.R, (int *)tasks_am, P.d_jtab, msg);
            if (rc != SPN_OK) return set_err(rc, msg);
        }
        if (argmax && !P.jfused_argmax) {
            cudaError_t e = argmax_rows_launch(out, n, P.R, argmax, (cudaStream_t)stream);
            if (e != cudaSuccess) return cuda_err(e, "argmax launch");
        }
        return SPN_OK;
    }
    if (P.path == 1 && P.r2) {
        R2Params rp = P.r2p;
        rp.xT = P.d_xT;
        rp.ldT = P.chunk;
        cudaError_t e;
        if (P.cert) {
            if (n > P.flag_cap) {  // room for every sample of this call
                if (P.d_flag_idx) cudaFreeAsync(P.d_flag_idx, (cudaStream_t)stream);
                P.d_flag_idx = nullptr;
                P.flag_cap = 0;
                if ((e = cudaMallocAsync((void **)&P.d_flag_idx, (size_t)n * 8, (cudaStream_t)stream)) !=
                    cudaSuccess)
                    return set_err(SPN_E_OOM, "certification index list");
                P.flag_cap = n;
            }
            if ((e = cudaMemsetAsync(P.d_flag_count, 0, sizeof(int32_t), (cudaStream_t)stream)) != cudaSuccess)
                return cuda_err(e, "cudaMemsetAsync");
            rp.flag_count = P.d_flag_count;
            rp.flag_idx = P.d_flag_idx;
            rp.cert_err = P.cert_err;
            // 0.9 of the north-star tolerance (1e-4): the remaining 0.1 covers the fp32
            // arithmetic both precisions share (measured 2.2e-7 relative on C4, hi/lo vs oracle)
            rp.cert_tol = 0.9e-4f;
        }
        // launch chunk: the transposed-scratch capacity, or (host pipeline)
        // smaller pieces that start as soon as their rows have landed
        const int64_t LC = lchunk > 0 ? std::min(lchunk, P.chunk) : P.chunk;
        for (int64_t c0 = 0; c0 < n; c0 += LC) {
            rp.row0 = c0;
            const int64_t m = std::min(LC, n - c0);
            const int64_t rows_pad = (m + 127) / 128 * 128;
            if (ready && (e = cudaStreamWaitEvent((cudaStream_t)stream, ready[c0 / LC], 0)) != cudaSuccess)
                return cuda_err(e, "cudaStreamWaitEvent");
            e = transpose_launch(x + c0 * ld, m, ld, P.F, P.d_xT, P.chunk, rows_pad,
                                 (cudaStream_t)stream);
            if (e != cudaSuccess) return cuda_err(e, "transpose launch");
            rp.n = m;
            rp.out = out + c0 * P.R;
            rp.argmax = argmax ? argmax + c0 : nullptr;
            const int grid = (int)std::min<int64_t>((m + 127) / 128, P.grid_max);
            e = rat2_launch(rp, P.d_r2leaf, P.n_r2leaf, P.d_r2sum, P.n_r2sum, marg, grid,
                            (cudaStream_t)stream);
            if (e != cudaSuccess) return cuda_err(e, "rat2 launch");
        }
        if (P.cert) {
            // flagged samples (count on the device): gather their rows into the
            // transposed scratch, v1 kernel in hi/lo precision, scatter back;
            // one round per chunk of capacity, each a no-op when nothing is left
            RParams vp = v1_params(P);
            vp.xT = P.d_xT;
            vp.ldT = P.chunk;
            vp.out = P.d_cert_out;
            vp.argmax = P.d_cert_am;
            vp.n = P.chunk;
            vp.n_count = P.d_flag_count;
            for (int64_t off = 0; off < n; off += P.chunk) {
                vp.n_off = off;
                if ((e = cert_gather_launch(x, ld, P.F, P.d_flag_idx, P.d_flag_count, off, P.chunk, P.d_xT,
                                            P.chunk, (cudaStream_t)stream)) != cudaSuccess)
                    return cuda_err(e, "certification gather");
                if ((e = rat_launch(vp, marg, P.grid_max, P.smem, (cudaStream_t)stream)) != cudaSuccess)
                    return cuda_err(e, "certification recompute");
                if ((e = cert_scatter_launch(P.d_cert_out, P.d_cert_am, P.d_flag_idx, P.d_flag_count, off,
                                             P.chunk, P.R, out, argmax, (cudaStream_t)stream)) != cudaSuccess)
                    return cuda_err(e, "certification scatter");
            }
        }
        return SPN_OK;
    }
    if (P.path == 1) {
        RParams rp = v1_params(P);
        rp.xT = P.d_xT;
        rp.ldT = P.chunk;
        for (int64_t c0 = 0; c0 < n; c0 += P.chunk) {
            const int64_t m = std::min(P.chunk, n - c0);
            const int64_t rows_pad = (m + 127) / 128 * 128;
            cudaError_t e = transpose_launch(x + c0 * ld, m, ld, P.F, P.d_xT, P.chunk, rows_pad,
                                             (cudaStream_t)stream);
            if (e != cudaSuccess) return cuda_err(e, "transpose launch");
            rp.n = m;
            rp.out = out + c0 * P.R;
            rp.argmax = argmax ? argmax + c0 : nullptr;
            const int grid = (int)std::min<int64_t>((m + 127) / 128, P.grid_max);
            e = rat_launch(rp, marg, grid, P.smem, (cudaStream_t)stream);
            if (e != cudaSuccess) return cuda_err(e, "rat_eval launch");
        }
        return SPN_OK;
    }
    KParams kp;
    memset(&kp, 0, sizeof(kp));
    kp.prog = P.d_prog;
    kp.task_off = P.d_task_off;
    kp.n_tasks = P.n_tasks;
    kp.prog_cap = P.prog_cap;
    kp.first_task_len = P.first_task_len;
    kp.tables = P.d_tables;
    kp.edges = P.d_edges;
    kp.x = x;
    kp.n = n;
    kp.ld = ld;
    kp.F = P.F;
    kp.R = P.R;
    kp.out = out;
    kp.argmax = argmax;
    kp.gslots = P.d_gslots;
    kp.n_gslots = (int32_t)P.n_gslots;
    kp.n_sslots = (int32_t)P.n_sslots;
    kp.x_in_smem = P.xs;
    kp.tpw = P.tpw;
    const int WT = 32 * P.K;
    kp.n_wtiles = (n + WT - 1) / WT;
    const int nwarps = P.block / 32;
    int64_t need;
    if (P.n_tasks == 1) need = (kp.n_wtiles + nwarps - 1) / nwarps;
    else need = (n + (int64_t)nwarps * WT - 1) / ((int64_t)nwarps * WT);
    const int grid = (int)std::max<int64_t>(1, std::min<int64_t>(need, P.grid_max));
    return launch_kernel(kp, P.K, marg, P.xs, grid, P.block, P.smem, (cudaStream_t)stream);
}

// Host pipeline of a certified layered v2 plan.  Its certification
// recomputes flagged samples with the v1 kernel, whose latency is about one
// 128-sample tile (~20 ms on C5) however few samples are flagged, so one
// round per transposed chunk (~46 ms of work) would cost ~40%.  Instead a
// whole group of host rows (up to ~4 GB of features) is kept on the device:
// the copy stream lands it chunk by chunk (an event per chunk), the compute
// stream starts each chunk as soon as its rows are in, and the group ends
// with one certification round and one copy of the outputs back.
int infer_host_grouped(DevicePlan &P, spn_handle *h, const float *x, int64_t n, int64_t ld,
                       float *out, int32_t *argmax, bool marg) {
    cudaError_t e;
    const int64_t per_chunk = P.chunk * P.F * 4;
    int64_t max_chunks = std::max<int64_t>(1, ((int64_t)4 << 30) / per_chunk);
    // SPNB_HOST_GROUP_CHUNKS (tests): smaller groups, to cover several groups per call
    if (const char *ev = getenv("SPNB_HOST_GROUP_CHUNKS")) max_chunks = std::max(1, atoi(ev));
    // groups as large as this call needs (up to ~4 GB of rows): (re)allocated
    // when a call needs more than the current buffers hold, halved while the
    // device is short of memory (down to one transposed chunk)
    const int64_t want = std::min<int64_t>(max_chunks, std::max<int64_t>(1, (n + P.chunk - 1) / P.chunk));
    if (!P.gx || want * P.chunk > P.group_cap) {
        if (P.gx) {
            for (int i = 0; i < 2; ++i) cudaStreamSynchronize(P.hs[i]);  // (an earlier call may have failed midway)
            cudaFree(P.gx);
            cudaFree(P.gout);
            cudaFree(P.gam);
            P.gx = nullptr;
            P.gout = nullptr;
            P.gam = nullptr;
            for (cudaEvent_t ev : P.gev) cudaEventDestroy(ev);
            P.gev.clear();
        }
        for (int64_t chunks = want;; chunks = (chunks + 1) / 2) {
            P.group_cap = chunks * P.chunk;
            if (cudaMalloc(&P.gx, (size_t)P.group_cap * P.F * 4) == cudaSuccess &&
                cudaMalloc(&P.gout, (size_t)P.group_cap * P.R * 4) == cudaSuccess &&
                cudaMalloc(&P.gam, (size_t)P.group_cap * 4) == cudaSuccess)
                break;
            cudaFree(P.gx);
            cudaFree(P.gout);
            cudaFree(P.gam);
            P.gx = nullptr;
            P.gout = nullptr;
            P.gam = nullptr;
            P.group_cap = 0;
            cudaGetLastError();  // clear the allocation error
            if (chunks == 1) return set_err(SPN_E_OOM, "host pipeline group buffers");
        }
        // copies and launches in pieces of one 128-sample tile per CTA, so the
        // first launch waits for ~1/8 of a transposed chunk, not all of it
        P.group_piece = std::max<int64_t>(128, P.chunk / 8 / 128 * 128);
        P.gev.resize((size_t)((P.group_cap + P.group_piece - 1) / P.group_piece), nullptr);
        for (auto &ev : P.gev)
            if ((e = cudaEventCreateWithFlags(&ev, cudaEventDisableTiming)) != cudaSuccess)
                return cuda_err(e, "cudaEventCreate");
        if (!P.gdone && (e = cudaEventCreateWithFlags(&P.gdone, cudaEventDisableTiming)) != cudaSuccess)
            return cuda_err(e, "cudaEventCreate");
    }
    cudaStream_t cp = P.hs[0], cs = P.hs[1];
    bool first = true;
    for (int64_t g0 = 0; g0 < n; g0 += P.group_cap) {
        const int64_t m = std::min(P.group_cap, n - g0);
        // the previous group's kernels and output copies are done with gx / gout
        if (!first && (e = cudaStreamWaitEvent(cp, P.gdone, 0)) != cudaSuccess)
            return cuda_err(e, "cudaStreamWaitEvent");
        first = false;
        for (int64_t c0 = 0; c0 < m; c0 += P.group_piece) {
            const int64_t mc = std::min(P.group_piece, m - c0);
            const float *src = x + (g0 + c0) * ld;
            if (ld == P.F)
                e = cudaMemcpyAsync(P.gx + c0 * P.F, src, (size_t)mc * P.F * 4, cudaMemcpyHostToDevice, cp);
            else
                e = cudaMemcpy2DAsync(P.gx + c0 * P.F, (size_t)P.F * 4, src, (size_t)ld * 4,
                                      (size_t)P.F * 4, (size_t)mc, cudaMemcpyHostToDevice, cp);
            if (e != cudaSuccess) return cuda_err(e, "H2D");
            if ((e = cudaEventRecord(P.gev[(size_t)(c0 / P.group_piece)], cp)) != cudaSuccess)
                return cuda_err(e, "cudaEventRecord");
        }
        int rc;
        {
            // same scratch ordering as infer_device (another stream's call may still use it)
            std::lock_guard<std::mutex> lk(P.scratch_mu);
            if (P.scratch_ev && P.scratch_stream != (void *)cs &&
                (e = cudaStreamWaitEvent(cs, P.scratch_ev, 0)) != cudaSuccess)
                return cuda_err(e, "cudaStreamWaitEvent");
            rc = infer_device_impl(h, P.gx, m, P.F, P.gout, argmax ? P.gam : nullptr, cs, marg,
                                   P.gev.data(), P.group_piece);
            if (rc != SPN_OK) return rc;
            if (!P.scratch_ev &&
                (e = cudaEventCreateWithFlags(&P.scratch_ev, cudaEventDisableTiming)) != cudaSuccess)
                return cuda_err(e, "cudaEventCreate");
            if ((e = cudaEventRecord(P.scratch_ev, cs)) != cudaSuccess) return cuda_err(e, "cudaEventRecord");
            P.scratch_stream = cs;
        }
        if ((e = cudaMemcpyAsync(out + g0 * P.R, P.gout, (size_t)m * P.R * 4, cudaMemcpyDeviceToHost, cs)) !=
            cudaSuccess)
            return cuda_err(e, "D2H");
        if (argmax && (e = cudaMemcpyAsync(argmax + g0, P.gam, (size_t)m * 4, cudaMemcpyDeviceToHost, cs)) !=
                          cudaSuccess)
            return cuda_err(e, "D2H argmax");
        if ((e = cudaEventRecord(P.gdone, cs)) != cudaSuccess) return cuda_err(e, "cudaEventRecord");
    }
    for (int i = 0; i < 2; ++i)
        if ((e = cudaStreamSynchronize(P.hs[i])) != cudaSuccess) return cuda_err(e, "sync");
    return SPN_OK;
}

int infer_host(spn_handle *h, const float *x, int64_t n, int64_t ld, float *out, int32_t *argmax,
               bool marg) {
    if (!h || h->magic != H_PLAN) return set_err(SPN_E_ARG, "not a plan handle");
    DevicePlan &P = *h->plan;
    if (n < 0) return set_err(SPN_E_ARG, "n < 0");
    if (n == 0) return SPN_OK;
    if (!x || !out) return set_err(SPN_E_ARG, "null x/out");
    if (ld < P.F) return set_err(SPN_E_ARG, "ld < n_features");
    std::lock_guard<std::mutex> lk(P.host_mu);
    DeviceGuard dg(P.device);
    cudaError_t e;
    const bool grouped = P.path == 1 && P.r2 && P.cert;
    if (!P.hs[0]) {
        // chunk sized to ~32 MB of features: big enough to amortise launches,
        // small enough to overlap H2D / kernel / D2H across the two streams
        P.host_chunk = std::max<int64_t>(4096, ((int64_t)(32 << 20) / (4 * P.F)) & ~int64_t(4095));
        // the layered path launches one persistent wave per transposed chunk:
        // host chunks of that size keep every SM busy (C5: 151,552 samples)
        if (P.path == 1) P.host_chunk = std::max<int64_t>(P.host_chunk, P.chunk);
        for (int i = 0; i < 2; ++i) {
            if ((e = cudaStreamCreateWithFlags(&P.hs[i], cudaStreamNonBlocking)) != cudaSuccess)
                return cuda_err(e, "cudaStreamCreate");
            if (grouped) continue;  // infer_host_grouped allocates its own buffers
            if ((e = cudaMalloc(&P.hx[i], (size_t)P.host_chunk * P.F * 4)) != cudaSuccess ||
                (e = cudaMalloc(&P.hout[i], (size_t)P.host_chunk * P.R * 4)) != cudaSuccess ||
                (e = cudaMalloc(&P.ham[i], (size_t)P.host_chunk * 4)) != cudaSuccess)
                return set_err(SPN_E_OOM, "host pipeline buffers");
        }
    }
    if (grouped) return infer_host_grouped(P, h, x, n, ld, out, argmax, marg);
    const int64_t C = P.host_chunk;
    int rc = SPN_OK;
    for (int64_t c0 = 0, i = 0; c0 < n; c0 += C, ++i) {
        const int s = (int)(i & 1);
        const int64_t m = std::min(C, n - c0);
        cudaStream_t st = P.hs[s];
        if (ld == P.F)  // contiguous rows: one linear copy (2-D copies of 104-byte rows are slow)
            e = cudaMemcpyAsync(P.hx[s], x + c0 * ld, (size_t)m * P.F * 4, cudaMemcpyHostToDevice, st);
        else
            e = cudaMemcpy2DAsync(P.hx[s], (size_t)P.F * 4, x + c0 * ld, (size_t)ld * 4,
                                  (size_t)P.F * 4, (size_t)m, cudaMemcpyHostToDevice, st);
        if (e != cudaSuccess) return cuda_err(e, "H2D");
        rc = infer_device(h, P.hx[s], m, P.F, P.hout[s], argmax ? P.ham[s] : nullptr, st, marg);
        if (rc != SPN_OK) return rc;
        e = cudaMemcpyAsync(out + c0 * P.R, P.hout[s], (size_t)m * P.R * 4,
                            cudaMemcpyDeviceToHost, st);
        if (e != cudaSuccess) return cuda_err(e, "D2H");
        if (argmax) {
            e = cudaMemcpyAsync(argmax + c0, P.ham[s], (size_t)m * 4, cudaMemcpyDeviceToHost, st);
            if (e != cudaSuccess) return cuda_err(e, "D2H argmax");
        }
    }
    for (int i = 0; i < 2; ++i)
        if ((e = cudaStreamSynchronize(P.hs[i])) != cudaSuccess) return cuda_err(e, "sync");
    return SPN_OK;
}

bool valid_graph_handle(const spn_handle *h) { return h && h->magic == H_GRAPH && h->graph; }

int prepare_layered(const GraphData &g, const LayeredPlan &lp, const spn_prepare_options &opt,
                    int dev, int sms, size_t smem, int wbufs,
                    std::chrono::steady_clock::time_point t0, spn_handle **out_plan) {
    DevicePlan *P = new (std::nothrow) DevicePlan();
    if (!P) return set_err(SPN_E_OOM, "plan");
    P->device = dev;
    P->path = 1;
    P->F = g.F;
    P->R = lp.C;
    P->sms = sms;
    P->smem = smem;
    P->grid_max = sms;
    P->block = 256;
    P->n_steps = (int32_t)lp.steps.size();
    P->prec = opt.tc_precision == 1 ? 1 : 3;
    P->smem_floats = lp.smem_floats;
    P->max_kpad = lp.max_kpad;
    P->max_ngroup = lp.max_ngroup;
    P->max_na = lp.max_na;
    P->max_vars = lp.max_vars;
    P->first_leaf = lp.first_leaf;
    P->max_leaf_params = lp.max_leaf_params;
    P->wbufs = wbufs;
    if (const char *ev = getenv("SPNB_TMEM_OVERLAP")) P->tmem_overlap = atoi(ev) != 0;
    // transposed-feature scratch: chunks small enough (<= ~48 MB) that the
    // tile slices re-read by every repetition stay resident in L2
    // (a multiple of one full wave of 128-sample tiles: 148 SMs x 128)
    const int64_t wave = (int64_t)sms * 128;
    int64_t chunk = std::max<int64_t>(1, (((int64_t)48 << 20) / ((int64_t)g.F * 4)) / wave) * wave;
    P->chunk = chunk;
    int rc;
    std::vector<uint8_t> w8(lp.wimg.size() * 2);
    if (!w8.empty()) memcpy(w8.data(), lp.wimg.data(), w8.size());
    if ((rc = upload(&P->d_steps, lp.steps)) || (rc = upload(&P->d_vars, lp.vars)) ||
        (rc = upload(&P->d_fparams, lp.fparams)) || (rc = upload(&P->d_wimg, w8)) ||
        (rc = upload(&P->d_root_map, lp.root_map))) {
        free_plan(P);
        return rc;
    }
    if (getenv("SPNB_PROFILE") && cudaMalloc(&P->d_prof, 32 * sizeof(unsigned long long)) == cudaSuccess)
        cudaMemset(P->d_prof, 0, 32 * sizeof(unsigned long long));
    // ---- v2 kernel (rat2.cu): SPNB_RAT2=0 keeps the v1 kernel (A/B)
    int want_r2 = opt.layered_kernel;  // SPNB_RAT2 overrides auto (A/B experiments)
    if (const char *r2env = getenv("SPNB_RAT2"); r2env && want_r2 == 0) want_r2 = atoi(r2env) == 0 ? 1 : 0;
    if (want_r2 != 1) {
        Rat2Plan r2;
        // tensor-core leaves (opt-in, leaf_tc 2): measured slower than the FMA
        // leaves on C4 / C5, so auto keeps the FMA leaves;
        // they need the certification (it recomputes the inputs outside the
        // split operands' range)
        const bool try_ltc = opt.leaf_tc == 2;
        std::string ltc_why;
        if (try_ltc) {
            build_rat2(lp, r2, true);
            if (r2.ok && !std::isfinite(r2.tc_err_1pass)) {
                r2.ok = false;
                r2.why = "no certification bound (a zero sum weight)";
            }
            if (!r2.ok) ltc_why = r2.why;
        }
        if (opt.leaf_tc == 2 && (!r2.ok || opt.tc_precision != 0)) {
            free_plan(P);
            return set_err(SPN_E_UNSUPPORTED, opt.tc_precision != 0
                                                  ? std::string("leaf_tc 2 needs tc_precision 0 (certified)")
                                                  : "leaf_tc not applicable: " + ltc_why);
        }
        if (!r2.ok) build_rat2(lp, r2);
        if (r2.ok && !rat2_supported_shape(r2.I, r2.S)) {
            r2.ok = false;
            r2.why = "no v2 kernel instance for I = " + std::to_string(r2.I) + ", S = " +
                     std::to_string(r2.S);
        }
        int smem_optin = 0;
        cudaDeviceGetAttribute(&smem_optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
        R2Params rp;
        memset(&rp, 0, sizeof(rp));
        bool fits = false;
        // deepest rings that fit: leaf inputs 3..2, weight groups 3..2 (the
        // MMA warp holds a pair at once); the left/right leaf outputs have
        // R2_NAB = 3 slots (the leaf warps' run-ahead past the epilogue)
        static const int kRings[][2] = {{3, 3}, {3, 2}, {2, 3}, {2, 2}, {2, 2}};
        // tensor-core leaves: two input slots (features + parameter image)
        static const int kRingsT[][2] = {{2, 3}, {2, 2}, {2, 2}, {2, 2}, {2, 2}};
        const bool ltc = r2.ok && r2.leaf_tc;
        // v2 runs the single f16 pass (hi/lo operands do not fit its shared
        // memory on C4/C5-sized regions): tc_precision 2 keeps v1
        if (r2.ok && opt.tc_precision == 2) {
            r2.ok = false;
            r2.why = "tc_precision 2 (hi/lo) runs on the v1 kernel";
        }
        // SPNB_R2_RINGS=n_in,n_w (development): try these ring depths first
        if (const char *ev = getenv("SPNB_R2_RINGS"); ev && r2.ok && !ltc) {
            int ni = 0, nw = 0;
            if (sscanf(ev, "%d,%d", &ni, &nw) == 2 && ni >= 2 && ni <= 4 && nw >= 2 && nw <= 8)
                fits = rat2_layout(rp, r2.I, r2.max_vars, r2.max_blk, r2.kpad_bot, r2.kpad_up,
                                   r2.max_wgroup, 1, ni, nw, 0, 0, 0) <= smem_optin;
        }
        for (int a = 0; r2.ok && a < 5 && !fits; ++a)
            fits = rat2_layout(rp, r2.I, r2.max_vars, r2.max_blk, r2.kpad_bot, r2.kpad_up,
                               r2.max_wgroup, 1, ltc ? kRingsT[a][0] : kRings[a][0],
                               ltc ? kRingsT[a][1] : kRings[a][1], ltc ? r2.lvp : 0, r2.kl_j,
                               r2.kl_m) <= smem_optin;
        if (ltc && !fits && opt.leaf_tc != 2) {  // FMA leaves fit in less shared memory
            build_rat2(lp, r2);
            for (int a = 0; r2.ok && a < 5 && !fits; ++a)
                fits = rat2_layout(rp, r2.I, r2.max_vars, r2.max_blk, r2.kpad_bot, r2.kpad_up,
                                   r2.max_wgroup, 1, kRings[a][0], kRings[a][1], 0, 0, 0) <= smem_optin;
        }
        if (opt.leaf_tc == 2 && !(r2.ok && r2.leaf_tc && fits)) {
            free_plan(P);
            return set_err(SPN_E_UNSUPPORTED, "leaf_tc not applicable: shared memory");
        }
        if (r2.ok && fits) {
            std::vector<int32_t> leaf_idx, sum_idx;
            for (int32_t t = 0; t < (int32_t)r2.steps.size(); ++t)
                (r2.steps[t].type == 0 ? leaf_idx : sum_idx).push_back(t);
            std::vector<uint8_t> w2(r2.wimg.size() * 2);
            if (!w2.empty()) memcpy(w2.data(), r2.wimg.data(), w2.size());
            if ((rc = upload(&P->d_r2steps, r2.steps)) || (rc = upload(&P->d_r2vars, r2.vars)) ||
                (rc = upload(&P->d_r2fp, r2.fparams)) || (rc = upload(&P->d_r2w, w2)) ||
                (rc = upload(&P->d_r2rm, r2.root_map)) || (rc = upload(&P->d_r2leaf, leaf_idx)) ||
                (rc = upload(&P->d_r2sum, sum_idx))) {
                free_plan(P);
                return rc;
            }
            rp.steps = P->d_r2steps;
            rp.n_steps = (int32_t)r2.steps.size();
            rp.C = r2.C;
            rp.I = r2.I;
            rp.S = r2.S;
            rp.vars = P->d_r2vars;
            rp.fparams = P->d_r2fp;
            rp.wimg = P->d_r2w;
            rp.root_map = P->d_r2rm;
            rp.prec = 1;
            rp.max_vars = r2.max_vars;
            rp.max_blk = r2.max_blk;
            rp.kpad_bot = r2.kpad_bot;
            rp.kpad_up = r2.kpad_up;
            rp.max_wgroup = r2.max_wgroup;
            rp.gcols = r2.gcols;
            rp.D = r2.D;
            rp.prof = P->d_prof;
            P->r2p = rp;
            P->r2 = true;
            // auto precision: certify every sample's single-pass result against
            // the a-priori bound; failures are recomputed by v1 in hi/lo
            P->cert = opt.tc_precision == 0 && std::isfinite(r2.tc_err_1pass);
            P->cert_err = (float)r2.tc_err_1pass;
            P->n_r2leaf = (int32_t)leaf_idx.size();
            P->leaf_tc = r2.leaf_tc;
            P->n_r2sum = (int32_t)sum_idx.size();
            // (P->smem stays the v1 kernel's: it serves the certification fallback)
            // persistent kernel over many tiles per launch: 8 tiles per CTA
            chunk = (int64_t)sms * 128 * 8;
            P->chunk = chunk;
            if (P->cert && (cudaMalloc(&P->d_flag_count, sizeof(int32_t)) != cudaSuccess ||
                            cudaMalloc(&P->d_cert_out, (size_t)4 * chunk * lp.C) != cudaSuccess ||
                            cudaMalloc(&P->d_cert_am, (size_t)4 * chunk) != cudaSuccess)) {
                free_plan(P);
                return set_err(SPN_E_OOM, "certification buffers");
            }
        } else if (want_r2 == 2) {
            free_plan(P);
            return set_err(SPN_E_UNSUPPORTED, "layered v2 kernel not applicable: " +
                                                  (r2.ok ? std::string("shared memory") : r2.why));
        }
    }
    if (!P->r2 && (lp.w_max >= 32768.0 || (lp.w_min_nz > 0.0 && lp.w_min_nz < 0x1p-24))) {
        // v1 keeps weights unscaled in f16: out of range -> not this path
        free_plan(P);
        return set_err(SPN_E_UNSUPPORTED, "layered v1 kernel: sum weights outside the f16 range");
    }
    cudaError_t e = cudaMalloc(&P->d_xT, (size_t)g.F * chunk * 4);
    if (e != cudaSuccess) {
        free_plan(P);
        return set_err(SPN_E_OOM, "transposed feature scratch");
    }
    spn_plan_stats &s = P->stats;
    memset(&s, 0, sizeof(s));
    CGraph c;
    canonicalise(g, c);
    s.n_nodes = c.n;
    for (int64_t u = 0; u < c.n; ++u) {
        if (c.kind[u] == SPN_SUM) {
            s.n_sums++;
            s.n_sum_edges += c.cb[u + 1] - c.cb[u];
            s.mufu_per_sample += c.cb[u + 1] - c.cb[u] > 1 ? c.cb[u + 1] - c.cb[u] : 0;
        } else if (c.kind[u] == SPN_PRODUCT) {
            s.n_products++;
        } else {
            s.n_leaves++;
        }
    }
    // the layered path does not partition: one task; n_records = schedule steps
    s.n_tasks = 1;
    s.n_records = (int64_t)lp.steps.size();
    s.fma_per_sample = lp.fma_per_sample;
    s.mufu_per_sample = lp.mufu_per_sample;
    s.tc_flops_per_sample = lp.tc_flops_per_sample;  // algorithmic (one pass)
    if (P->r2 && P->leaf_tc) {
        // the leaf layer moved from the FMA pipe (2 per variable and
        // distribution) to the tensor cores (one GEMM of K = 2V + 1 per region)
        for (const LStep &st : lp.steps)
            if (st.type == 0) {
                s.fma_per_sample -= 2LL * st.n_out * st.n_vars;
                s.tc_flops_per_sample += 2LL * st.n_out * (2LL * st.n_vars + 1);
            }
    }
    s.bytes_per_sample = 4 * (int64_t)g.F + 4 * (int64_t)lp.C + 4;
    s.path = 1;
    s.chunk_samples = chunk;
    s.block_threads = P->r2 ? 512 : (lp.max_na > 48 ? 256 : 512);
    s.samples_per_thread = 0;
    s.grid = P->grid_max;
    s.smem_bytes = (int32_t)(P->r2 ? P->r2p.smem_bytes : P->smem);
    s.x_in_smem = 0;
    s.layered_kernel = P->r2 ? 2 : 1;
    s.tc_passes = P->r2 ? 1 : (P->prec == 3 ? 3 : 1);
    s.cert_err = P->r2 ? P->cert_err : 0.0;
    s.certified = P->cert ? 1 : 0;
    s.leaf_tc = P->r2 && P->leaf_tc ? 1 : 0;
    s.prepare_ms =
        std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
    spn_handle *h = new (std::nothrow) spn_handle();
    if (!h) {
        free_plan(P);
        return set_err(SPN_E_OOM, "handle");
    }
    h->magic = H_PLAN;
    h->plan = P;
    *out_plan = h;
    return SPN_OK;
}

// Compiled path (kernel KS): generate one straight-line kernel per task
// (codegen.cpp, emitted as PTX), assemble them for the device's architecture in
// parallel threads, load them with the driver API.  Returns SPN_OK with
// *out_plan set, or an error (the caller decides whether to fall back to
// the interpreter).
int prepare_compiled(const GraphData &g, const spn_prepare_options &opt, int dev, int sms,
                     std::chrono::steady_clock::time_point t0, spn_handle **out_plan) {
    JitOptions jo;
    jo.block = opt.block_threads ? opt.block_threads : 768;
    jo.space = opt.value_space;
    if (jo.block % 32 || jo.block < 32 || jo.block > 1024)
        return set_err(SPN_E_ARG, "block_threads must be a multiple of 32 in [32, 1024]");
    // launch bound: 768 resident threads per SM (<= 80 registers).  Default
    // one CTA of 768 threads: with the barrier-synchronised body (bar_every)
    // all 24 warps of the SM walk the same stretch of code.  Measured on C2
    // joint: 1 x 768 3.65e9 samples/s, 1 x 640 3.46e9, 1 x 1024 3.36e9,
    // 3 x 256 3.27e9, 1 x 512 3.25e9; marginal 1 x 768 2.56e9 vs 3 x 256
    // (spill fallback to 2 x 256) 2.12e9
    jo.min_blocks = opt.ctas_per_sm > 0 ? opt.ctas_per_sm : std::max(1, 768 / jo.block);
    if (const char *e = getenv("SPNB_JIT_MINB")) jo.min_blocks = std::max(1, atoi(e));
    // tiny SPNs (C1's toy: 12 nodes) are bound by HBM, not by their few
    // instructions: four interleaved samples per thread keep 4x the loads in
    // flight (large SPNs stay at one: register pressure, SPNB_JIT_K=2 measured
    // 1.42e9 vs 3.6e9 samples/s on C2)
    if ((int64_t)g.kind.size() <= 64) jo.samples_per_thread = 4;
    if (const char *e = getenv("SPNB_JIT_K")) jo.samples_per_thread = std::min(4, std::max(1, atoi(e)));
    // SPNB_JIT_TASKCAP (development): pack connected components up to this many nodes per kernel
    if (const char *e = getenv("SPNB_JIT_TASKCAP")) jo.task_cap_nodes = std::max<int64_t>(1, atoll(e));
    if (const char *e = getenv("SPNB_JIT_BAR")) jo.bar_every = std::max(0, atoi(e));
    JitProgram jp;
    std::string msg;
    int rc = generate_jit(g, jo, jp, msg);
    if (rc != SPN_OK) return set_err(rc, msg);
    if (opt.compiled_path == 0)
        for (const JitTask &t : jp.tasks)
            if (t.max_live > jo.max_live_auto)
                return set_err(SPN_E_UNSUPPORTED, "compiled path: " + std::to_string(t.max_live) +
                                                      " values live at once in " + t.name +
                                                      " (auto limit " +
                                                      std::to_string(jo.max_live_auto) + ")");
    int major = 0, minor = 0;
    cudaDeviceGetAttribute(&major, cudaDevAttrComputeCapabilityMajor, dev);
    cudaDeviceGetAttribute(&minor, cudaDevAttrComputeCapabilityMinor, dev);
    if (major < 10) return set_err(SPN_E_UNSUPPORTED, "compiled path targets sm_100a (B200)");
    const std::string arch = std::to_string(major * 10 + minor) + "a";
    const auto tc0 = std::chrono::steady_clock::now();
    const size_t T = jp.tasks.size();
    // 2T assembly jobs (joint + marginal module per task) on all host cores
    std::vector<std::vector<char>> cubins(2 * T);
    std::vector<std::string> logs(2 * T);
    std::vector<int> rcs(2 * T, SPN_OK);
    {
        const size_t J = 2 * T;
        const size_t nthreads = std::max<size_t>(1, std::min<size_t>(J, std::thread::hardware_concurrency()));
        std::atomic<size_t> next{0};
        std::vector<std::thread> th;
        for (size_t i = 0; i < nthreads; ++i)
            th.emplace_back([&] {
                for (size_t j; (j = next++) < J;)
                    rcs[j] = jit_compile(jp.tasks[j / 2].ptx[j % 2], arch, cubins[j], logs[j]);
            });
        for (auto &x : th) x.join();
    }
    for (size_t j = 0; j < 2 * T; ++j)
        if (rcs[j] != SPN_OK) return set_err(rcs[j], "compiled path: " + logs[j].substr(0, 2000));
    const double compile_ms =
        std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - tc0).count();
    DevicePlan *P = new (std::nothrow) DevicePlan();
    if (!P) return set_err(SPN_E_OOM, "plan");
    P->device = dev;
    P->path = 2;
    P->F = g.F;
    P->R = (int32_t)g.roots.size();
    P->sms = sms;
    P->jblock = jo.block;
    P->jK = jo.samples_per_thread;
    P->jfused_argmax = jp.fused_argmax;
    P->block = jo.block;
    int max_regs = 0, min_occ = 1 << 30;
    for (size_t t = 0; t < T; ++t) {
        P->jk.push_back(JitKernel());
        JitKernel &k = P->jk.back();
        for (int v = 0; v < 2; ++v) {
            if ((rc = jit_load(cubins[2 * t + v], jp.tasks[t].name, v, jo.block, k, msg)) != SPN_OK) {
                free_plan(P);
                return set_err(rc, msg);
            }
            // auto launch bounds: a variant that spills at min_blocks CTAs/SM
            // is regenerated with one CTA/SM fewer (measured on C2: the
            // marginal kernel spills 720 B at 3 x 256 threads, 80 registers,
            // and runs 11% slower than at 2 x 256 without spills)
            for (int mb = jo.min_blocks - 1; k.local_bytes[v] > 0 && opt.ctas_per_sm <= 0 && mb >= 1; --mb) {
                JitOptions jo2 = jo;
                jo2.min_blocks = mb;
                JitProgram jp2;
                std::vector<char> cb;
                std::string log;
                if (generate_jit(g, jo2, jp2, msg) != SPN_OK ||
                    jit_compile(jp2.tasks[t].ptx[v], arch, cb, log) != SPN_OK)
                    break;
                JitKernel k2;
                if (jit_load(cb, jp2.tasks[t].name, v, jo.block, k2, msg) != SPN_OK) break;
                jit_unload_variant(k, v);
                k.module[v] = k2.module[v];
                k.fn[v] = k2.fn[v];
                k.regs[v] = k2.regs[v];
                k.occupancy[v] = k2.occupancy[v];
                k.local_bytes[v] = k2.local_bytes[v];
                k.block[v] = k2.block[v];
            }
            // (a variant still spilling at one CTA of 768 threads keeps it:
            // regenerating the C2 marginal kernel with 512-thread CTAs, no
            // spills, measured 2.20e9 vs 2.57e9 samples/s; 640 threads 2.59e9)
        }
        // grid-stride loop over samples with exactly one wave of resident CTAs
        // (per variant): every thread gets ceil or floor of n / threads samples
        // (measured on C2: 4 waves left SMs idle for up to one extra iteration)
        const int occ = std::max(1, std::min(k.occupancy[0], k.occupancy[1]));
        P->jgrid_max.push_back(sms * std::max(1, k.occupancy[0]));
        P->jgrid_max_m.push_back(sms * std::max(1, k.occupancy[1]));
        max_regs = std::max({max_regs, k.regs[0], k.regs[1]});
        min_occ = std::min(min_occ, occ);
    }
    if ((rc = upload(&P->d_jtab, jp.tables))) {
        free_plan(P);
        return rc;
    }
    spn_plan_stats &s = P->stats;
    memset(&s, 0, sizeof(s));
    s.n_nodes = jp.n_nodes;
    s.n_leaves = jp.n_leaves;
    s.n_sums = jp.n_sums;
    s.n_products = jp.n_products;
    s.n_sum_edges = jp.n_sum_edges;
    s.n_tasks = (int64_t)T;
    s.mufu_per_sample = jp.mufu_per_sample;
    s.fma_per_sample = jp.fma_per_sample;
    s.bytes_per_sample = 4 * (int64_t)g.F + 4 * (int64_t)g.roots.size();
    s.path = 2;
    s.block_threads = jo.block;
    s.samples_per_thread = jo.samples_per_thread;
    s.grid = P->jgrid_max.empty() ? 0 : P->jgrid_max[0];
    s.x_in_smem = 0;
    s.kernel_regs = max_regs;
    s.ctas_per_sm = min_occ;
    s.mufu_exec_per_sample = jp.mufu_exec_per_sample;
    s.value_space = jp.linear ? 2 : 1;
    s.compile_ms = compile_ms;
    s.prepare_ms =
        std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
    spn_handle *h = new (std::nothrow) spn_handle();
    if (!h) {
        free_plan(P);
        return set_err(SPN_E_OOM, "handle");
    }
    h->magic = H_PLAN;
    h->plan = P;
    *out_plan = h;
    return SPN_OK;
}

}  // namespace

extern "C" {

void spn_default_options(spn_prepare_options *opt) {
    if (!opt) return;
    memset(opt, 0, sizeof(*opt));
    opt->device = -1;
}

const char *spn_last_error(void) { return t_err.c_str(); }

int spn_load_graph(const spn_node *nodes, int64_t n_nodes, const int64_t *children,
                   const double *weights, int64_t n_edges, const double *params,
                   int64_t n_params, const int64_t *roots, int32_t n_roots, int32_t n_features,
                   spn_handle **out_graph) {
    if (!out_graph) return set_err(SPN_E_ARG, "out_graph is NULL");
    *out_graph = nullptr;
    if (n_nodes < 0 || n_edges < 0 || n_params < 0 || n_roots < 1 || n_features < 1)
        return set_err(SPN_E_ARG, "negative size, n_roots < 1 or n_features < 1");
    if ((n_nodes && !nodes) || (n_edges && (!children || !weights)) || (n_params && !params) ||
        !roots)
        return set_err(SPN_E_ARG, "null array with non-zero size");
    GraphData *g = new (std::nothrow) GraphData();
    if (!g) return set_err(SPN_E_OOM, "graph allocation");
    try {
        g->F = n_features;
        g->kind.resize(n_nodes);
        g->feature.resize(n_nodes);
        g->n_children.resize(n_nodes);
        g->n_params.resize(n_nodes);
        g->child_begin.resize(n_nodes);
        g->param_begin.resize(n_nodes);
        for (int64_t i = 0; i < n_nodes; ++i) {
            g->kind[i] = nodes[i].kind;
            g->feature[i] = nodes[i].feature;
            g->n_children[i] = nodes[i].n_children;
            g->n_params[i] = nodes[i].n_params;
            g->child_begin[i] = nodes[i].child_begin;
            g->param_begin[i] = nodes[i].param_begin;
        }
        g->children.assign(children, children + n_edges);
        g->weights.assign(weights, weights + n_edges);
        g->params.assign(params, params + n_params);
        g->roots.assign(roots, roots + n_roots);
    } catch (...) {
        delete g;
        return set_err(SPN_E_OOM, "graph copy");
    }
    std::string msg;
    const int rc = validate_graph(*g, msg);
    if (rc != SPN_OK) {
        delete g;
        return set_err(rc, msg);
    }
    spn_handle *h = new (std::nothrow) spn_handle();
    if (!h) {
        delete g;
        return set_err(SPN_E_OOM, "handle");
    }
    h->magic = H_GRAPH;
    h->graph = g;
    *out_graph = h;
    return SPN_OK;
}

int spn_prepare(const spn_handle *graph, const spn_prepare_options *opt_in,
                spn_handle **out_plan) {
    if (!out_plan) return set_err(SPN_E_ARG, "out_plan is NULL");
    *out_plan = nullptr;
    if (!valid_graph_handle(graph)) return set_err(SPN_E_ARG, "not a graph handle");
    spn_prepare_options opt;
    spn_default_options(&opt);
    if (opt_in) opt = *opt_in;
    for (int i = 0; i < 4; ++i)
        if (opt.reserved[i]) return set_err(SPN_E_ARG, "reserved option fields must be zero");
    if (opt.leaf_tc < 0 || opt.leaf_tc > 2)
        return set_err(SPN_E_ARG, "leaf_tc must be 0 (auto), 1 (off) or 2 (force)");
    if (opt.value_space < 0 || opt.value_space > 2)
        return set_err(SPN_E_ARG, "value_space must be 0 (auto), 1 (log2) or 2 (linear)");
    if (opt.value_space == 2 && (opt.compiled_path == 1 || opt.layered_path == 2))
        return set_err(SPN_E_ARG, "value_space 2 (linear) needs the compiled path");
    if (opt.layered_kernel < 0 || opt.layered_kernel > 2)
        return set_err(SPN_E_ARG, "layered_kernel must be 0 (auto), 1 (v1) or 2 (v2)");
    if (opt.compiled_path < 0 || opt.compiled_path > 2)
        return set_err(SPN_E_ARG, "compiled_path must be 0 (auto), 1 (off) or 2 (force)");
    const auto t0 = std::chrono::steady_clock::now();
    const GraphData &g = *graph->graph;

    int dev = opt.device;
    cudaError_t e;
    if (dev < 0 && (e = cudaGetDevice(&dev)) != cudaSuccess) return cuda_err(e, "cudaGetDevice");
    DeviceGuard dg(dev);
    int sms = 0, smem_optin = 0;
    if ((e = cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev)) != cudaSuccess)
        return cuda_err(e, "device attributes");
    cudaDeviceGetAttribute(&smem_optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);

    // ---- layered (RAT-SPN) tensor-core path ----
    if (opt.layered_path != 1 && opt.value_space != 2) {
        LayeredPlan lp;
        size_t lsmem = 0;
        int wbufs = 0;
        const int prec = opt.tc_precision == 1 ? 1 : 3;
        // weight-group buffering, first that fits in shared memory: N <= 240
        // or N <= 120 per group with double-buffered weights, then a single
        // buffer (measured on C4: a third buffer, prefetch distance 2, gave
        // no gain -- the ring code supports it; scripts/gpu/run_lay12.sh)
        static const int kAttempts[][2] = {{240, 2}, {120, 2}, {240, 1}, {120, 1}, {120, 1}};
        int first_attempt = 0;  // SPNB_LAYERED_ATTEMPT: index into kAttempts (A/B)
        if (const char *ev = getenv("SPNB_LAYERED_ATTEMPT")) first_attempt = std::min(4, std::max(0, atoi(ev)));
        for (int attempt = first_attempt; attempt < 5 && wbufs == 0; ++attempt) {
            const int n_cap = kAttempts[attempt][0];
            const int wb = kAttempts[attempt][1];
            detect_layered(g, lp, n_cap);
            if (!lp.ok) break;
            lsmem = rat_smem_bytes(lp.smem_floats, lp.C, lp.max_na, lp.max_kpad, lp.max_ngroup,
                                   lp.max_vars, lp.max_leaf_params, prec, wb);
            if (lsmem <= (size_t)smem_optin) wbufs = wb;
        }
        if (lp.ok && wbufs == 0) {
            lp.ok = false;
            lp.why = "activations do not fit in shared memory";
        }
        if (!lp.ok && opt.layered_path == 2)
            return set_err(SPN_E_UNSUPPORTED, "layered path not applicable: " + lp.why);
        if (lp.ok) {
            const int rc = prepare_layered(g, lp, opt, dev, sms, lsmem, wbufs, t0, out_plan);
            // auto: a layered graph neither kernel can serve goes to the generic path
            if (rc != SPN_E_UNSUPPORTED || opt.layered_path == 2) return rc;
        }
    }
    // ---- compiled path: one generated straight-line kernel per task ----
    // auto: used unless the caller pins interpreter parameters
    // (samples_per_thread / max_task_nodes) or a component is too large
    if (opt.compiled_path == 2 || opt.value_space == 2 ||
        (opt.compiled_path == 0 && opt.samples_per_thread == 0 && opt.max_task_nodes == 0)) {
        const int rc = prepare_compiled(g, opt, dev, sms, t0, out_plan);
        if (rc == SPN_OK || opt.compiled_path == 2 || opt.value_space == 2 || rc == SPN_E_ARG ||
            rc == SPN_E_OOM)
            return rc;
        // SPN_E_UNSUPPORTED / SPN_E_CUDA from the compiler or loader: the
        // interpreter kernel (also sm_100a, not a CPU path) serves the graph
    }
    // auto: K = 2 samples/thread with up to 24 warps when 16+ warps' feature
    // tiles fit in shared memory (more warps hide the interpreter's latency),
    // else K = 4 (measured on C2: K2x24 warps 0.733 ms vs K4x12 0.776 ms)
    int K = opt.samples_per_thread ? opt.samples_per_thread
                                   : ((size_t)g.F * 68 * 4 * 16 <= (size_t)170 * 1024 ? 2 : 4);
    if (K != 1 && K != 2 && K != 4 && K != 8)
        return set_err(SPN_E_ARG, "samples_per_thread must be 1, 2, 4 or 8");
    const int max_block = K == 8 ? 256 : (K == 4 ? 384 : (K == 2 ? 768 : 512));
    int block = opt.block_threads ? opt.block_threads : max_block;
    if (block % 32 || block < 32 || block > max_block)
        return set_err(SPN_E_ARG, "block_threads must be a multiple of 32 within the kernel bound");
    int nwarps = block / 32;
    const int WT = 32 * K;
    const int tpw = WT + 4;
    const size_t xtile = (size_t)g.F * tpw * 4;
    // stage features in shared memory when a few warps' tiles fit comfortably
    bool xs = xtile * 4 <= (size_t)smem_optin * 3 / 4;

    CodegenConfig cfg;
    cfg.K = K;
    cfg.maxd = (K == 8 || K == 2) ? 10 : MAXD;
    cfg.x_in_smem = xs;
    cfg.tpw = tpw;
    cfg.max_task_ops = opt.max_task_nodes > 0 ? opt.max_task_nodes : -1;
    cfg.smem_slot_cap = 0;
    const bool auto_cap = opt.max_task_nodes == 0;
    PlanProgram prog;
    std::string msg;
    size_t smem = 0;
    for (int iter = 0;; ++iter) {
        prog = PlanProgram();
        int rc = build_program(g, cfg, prog, msg);
        if (rc != SPN_OK) return set_err(rc, msg);
        auto smem_of = [&](int nw, int64_t sslots) {
            return (size_t)(prog.max_task_records + 2) * sizeof(Rec) +
                   (size_t)nw * ((xs ? xtile : 0) + (size_t)sslots * WT * 4);
        };
        smem = smem_of(nwarps, prog.n_sslots);
        if (smem <= (size_t)smem_optin) {
            // give left-over shared memory to task-local slots (one rebuild)
            const int64_t spare = ((int64_t)smem_optin - (int64_t)smem_of(nwarps, 0)) /
                                  ((int64_t)nwarps * WT * 4);
            if (prog.n_gslots > 0 && cfg.smem_slot_cap == 0 && spare > 0 && iter < 40) {
                cfg.smem_slot_cap = std::min<int64_t>(spare, 4096);
                continue;
            }
            break;
        }
        if (iter > 40) return set_err(SPN_E_UNSUPPORTED, "cannot fit the plan into shared memory");
        if (xs && nwarps > 4 && !opt.block_threads) {
            nwarps -= (nwarps > 8 ? 2 : 1);
            block = nwarps * 32;
            continue;
        }
        if (prog.n_sslots > 0 && cfg.smem_slot_cap > 0) {
            cfg.smem_slot_cap /= 2;
            continue;
        }
        if (!auto_cap && cfg.max_task_ops > 0 && opt.max_task_nodes > 0)
            return set_err(SPN_E_UNSUPPORTED, "max_task_nodes too large for shared memory");
        // partition (or partition finer) so one task's program fits
        int64_t total_ops = 0;
        for (int64_t u = 0; u < (int64_t)g.kind.size(); ++u) total_ops += g.n_children[u] * 2;
        const int64_t budget_rec =
            ((int64_t)smem_optin - (int64_t)nwarps * (xs ? (int64_t)xtile : 0)) / (int64_t)sizeof(Rec) - 8;
        if (budget_rec < 64) return set_err(SPN_E_UNSUPPORTED, "no shared memory left for the program");
        if (cfg.max_task_ops <= 0) cfg.max_task_ops = std::max<int64_t>(64, budget_rec / 2);
        else cfg.max_task_ops = std::max<int64_t>(32, cfg.max_task_ops * 2 / 3);
    }

    DevicePlan *P = new (std::nothrow) DevicePlan();
    if (!P) return set_err(SPN_E_OOM, "plan");
    P->device = dev;
    P->K = K;
    P->xs = xs;
    P->tpw = tpw;
    P->block = block;
    P->smem = smem;
    P->sms = sms;
    P->F = g.F;
    P->R = (int32_t)g.roots.size();
    P->n_tasks = (int32_t)(prog.task_off.size() - 1);
    P->first_task_len = (int32_t)(prog.task_off[1] - prog.task_off[0]);
    P->prog_cap = (int)(prog.max_task_records + 2);
    P->n_sslots = prog.n_sslots;
    P->n_gslots = prog.n_gslots;
    int rc;
    if ((rc = upload(&P->d_prog, prog.prog)) || (rc = upload(&P->d_task_off, prog.task_off)) ||
        (rc = upload(&P->d_tables, prog.tables)) || (rc = upload(&P->d_edges, prog.edges))) {
        free_plan(P);
        return rc;
    }
    int bps = occupancy(K, false, xs, block, smem);
    if (opt.ctas_per_sm > 0) bps = std::min(bps, opt.ctas_per_sm);
    if (bps < 1) {
        free_plan(P);
        return set_err(SPN_E_UNSUPPORTED, "kernel does not fit on an SM with this configuration");
    }
    P->grid_max = sms * bps;
    if (P->n_gslots > 0) {
        // per-warp scratch for values crossing tasks: a multi-task plan of a
        // very large SPN (C5 at <= 10k ops per task) keeps tens of thousands
        // of cut values live per sample, so the persistent grid is capped to
        // keep the scratch within 1/4 of free device memory (8 GiB at most);
        // the kernel's grid-stride loop covers any n with fewer warps
        size_t free_b = 0, total_b = 0;
        cudaMemGetInfo(&free_b, &total_b);
        const size_t budget = std::min<size_t>((size_t)8 << 30, free_b / 4);
        const size_t per_cta = (size_t)(block / 32) * P->n_gslots * WT * 4;
        P->grid_max = (int)std::max<size_t>(1, std::min<size_t>((size_t)P->grid_max, budget / per_cta));
        const size_t bytes = (size_t)P->grid_max * per_cta;
        if ((e = cudaMalloc(&P->d_gslots, bytes)) != cudaSuccess) {
            free_plan(P);
            return set_err(SPN_E_OOM, "scratch slots");
        }
    }
    spn_plan_stats &s = P->stats;
    memset(&s, 0, sizeof(s));
    s.n_nodes = prog.n_nodes;
    s.n_leaves = prog.n_leaves;
    s.n_sums = prog.n_sums;
    s.n_products = prog.n_products;
    s.n_sum_edges = prog.n_sum_edges;
    s.n_tasks = P->n_tasks;
    s.n_cut_values = prog.n_cut_values;
    s.partition_cost = prog.partition_cost;
    s.n_records = (int64_t)prog.prog.size();
    s.n_global_slots = prog.n_gslots;
    s.n_smem_slots = prog.n_sslots;
    s.max_stack = prog.max_stack;
    s.mufu_per_sample = prog.mufu_per_sample;
    s.fma_per_sample = prog.fma_per_sample;
    s.bytes_per_sample = 4 * (int64_t)g.F + 4 * (int64_t)g.roots.size();
    s.tc_flops_per_sample = 0;
    s.path = 0;
    s.block_threads = block;
    s.samples_per_thread = K;
    s.grid = P->grid_max;
    s.smem_bytes = (int32_t)smem;
    s.x_in_smem = xs;
    s.prepare_ms =
        std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
    spn_handle *h = new (std::nothrow) spn_handle();
    if (!h) {
        free_plan(P);
        return set_err(SPN_E_OOM, "handle");
    }
    h->magic = H_PLAN;
    h->plan = P;
    *out_plan = h;
    return SPN_OK;
}

int spn_infer_joint(spn_handle *plan, const float *x, int64_t n, int64_t ld, float *out,
                    int32_t *argmax, void *cuda_stream) {
    return infer_device(plan, x, n, ld, out, argmax, cuda_stream, false);
}

int spn_infer_marginal(spn_handle *plan, const float *x, int64_t n, int64_t ld, float *out,
                       int32_t *argmax, void *cuda_stream) {
    return infer_device(plan, x, n, ld, out, argmax, cuda_stream, true);
}

int spn_infer_joint_host(spn_handle *plan, const float *x, int64_t n, int64_t ld, float *out,
                         int32_t *argmax) {
    return infer_host(plan, x, n, ld, out, argmax, false);
}

int spn_infer_marginal_host(spn_handle *plan, const float *x, int64_t n, int64_t ld, float *out,
                            int32_t *argmax) {
    return infer_host(plan, x, n, ld, out, argmax, true);
}

int spn_plan_info(const spn_handle *plan, spn_plan_stats *stats) {
    if (!plan || plan->magic != H_PLAN || !stats) return set_err(SPN_E_ARG, "not a plan handle");
    *stats = plan->plan->stats;
    return SPN_OK;
}

int spn_partition_graph(const spn_handle *graph, int64_t max_task_ops, int32_t *task_of_node,
                        int32_t *n_tasks, int64_t *cost, int64_t *cut_values) {
    if (!valid_graph_handle(graph) || !task_of_node) return set_err(SPN_E_ARG, "bad arguments");
    std::vector<int32_t> t;
    PartitionResult res;
    const int rc = partition_graph(*graph->graph, max_task_ops, t, res);
    if (rc != SPN_OK) return set_err(rc, "partition failed");
    memcpy(task_of_node, t.data(), t.size() * sizeof(int32_t));
    if (n_tasks) *n_tasks = res.n_tasks;
    if (cost) *cost = res.cost;
    if (cut_values) *cut_values = res.cut_values;
    return SPN_OK;
}

int spn_build_program(const spn_handle *graph, int32_t samples_per_thread, int32_t x_in_smem,
                      int64_t max_task_ops, int64_t smem_slot_cap, void *records,
                      int64_t *n_records, int64_t *task_off, int64_t *n_tasks, float *tables,
                      int64_t *n_tables, void *edges, int64_t *n_edges, int64_t *slots) {
    if (!valid_graph_handle(graph) || !n_records || !n_tasks || !n_tables || !n_edges)
        return set_err(SPN_E_ARG, "bad arguments");
    if (samples_per_thread != 1 && samples_per_thread != 2 && samples_per_thread != 4 &&
        samples_per_thread != 8)
        return set_err(SPN_E_ARG, "samples_per_thread must be 1, 2, 4 or 8");
    CodegenConfig cfg;
    cfg.K = samples_per_thread;
    cfg.maxd = (samples_per_thread == 8 || samples_per_thread == 2) ? 10 : MAXD;
    cfg.x_in_smem = x_in_smem != 0;
    cfg.tpw = 32 * cfg.K + 4;
    cfg.max_task_ops = max_task_ops;
    cfg.smem_slot_cap = smem_slot_cap;
    PlanProgram prog;
    std::string msg;
    const int rc = build_program(*graph->graph, cfg, prog, msg);
    if (rc != SPN_OK) return set_err(rc, msg);
    const int64_t nr = (int64_t)prog.prog.size(), nt = (int64_t)prog.task_off.size() - 1;
    const int64_t ntab = (int64_t)prog.tables.size(), ne = (int64_t)prog.edges.size();
    if (records) {
        if (*n_records < nr || *n_tasks < nt || *n_tables < ntab || *n_edges < ne || !task_off ||
            !tables || !edges)
            return set_err(SPN_E_ARG, "buffers too small");
        memcpy(records, prog.prog.data(), nr * sizeof(Rec));
        memcpy(task_off, prog.task_off.data(), (nt + 1) * sizeof(int64_t));
        memcpy(tables, prog.tables.data(), ntab * sizeof(float));
        memcpy(edges, prog.edges.data(), ne * sizeof(Edge));
    }
    *n_records = nr;
    *n_tasks = nt;
    *n_tables = ntab;
    *n_edges = ne;
    if (slots) {
        slots[0] = prog.n_sslots;
        slots[1] = prog.n_gslots;
        slots[2] = prog.max_stack;
    }
    return SPN_OK;
}

int spn_build_layered2(const spn_handle *graph, int32_t *ok, char *why, int64_t why_len,
                       int64_t *sizes, int32_t *dims, void *steps, int32_t *vars, float *fparams,
                       void *wimg, int32_t *root_map, double *tc_err_1pass) {
    return spn_build_layered2_ex(graph, 0, ok, why, why_len, sizes, dims, steps, vars, fparams, wimg,
                                 root_map, tc_err_1pass);
}

int spn_build_layered2_ex(const spn_handle *graph, int32_t leaf_tc, int32_t *ok, char *why,
                          int64_t why_len, int64_t *sizes, int32_t *dims, void *steps, int32_t *vars,
                          float *fparams, void *wimg, int32_t *root_map, double *tc_err_1pass) {
    if (!valid_graph_handle(graph) || !ok || !sizes || !dims) return set_err(SPN_E_ARG, "bad arguments");
    LayeredPlan lp;
    detect_layered(*graph->graph, lp);
    Rat2Plan p;
    build_rat2(lp, p, leaf_tc != 0);
    *ok = p.ok ? 1 : 0;
    if (why && why_len > 0) {
        strncpy(why, p.why.c_str(), (size_t)why_len - 1);
        why[why_len - 1] = 0;
    }
    sizes[0] = (int64_t)p.steps.size();
    sizes[1] = (int64_t)p.vars.size();
    sizes[2] = (int64_t)p.fparams.size();
    sizes[3] = (int64_t)p.wimg.size() * 2;
    sizes[4] = (int64_t)p.root_map.size();
    sizes[5] = (int64_t)sizeof(R2Step);
    const int32_t d[14] = {p.F, p.C, p.I, p.S, p.D, p.gcols, p.kpad_bot, p.kpad_up,
                           p.max_wgroup, p.max_vars, p.max_blk, p.lvp, p.kl_j, p.kl_m};
    memcpy(dims, d, (leaf_tc ? 14 : 11) * sizeof(int32_t));
    if (tc_err_1pass) *tc_err_1pass = p.tc_err_1pass;
    if (steps) memcpy(steps, p.steps.data(), p.steps.size() * sizeof(R2Step));
    if (vars) memcpy(vars, p.vars.data(), p.vars.size() * 4);
    if (fparams) memcpy(fparams, p.fparams.data(), p.fparams.size() * 4);
    if (wimg) memcpy(wimg, p.wimg.data(), p.wimg.size() * 2);
    if (root_map) memcpy(root_map, p.root_map.data(), p.root_map.size() * 4);
    return SPN_OK;
}

int spn_build_layered(const spn_handle *graph, int32_t *is_layered, char *why, int64_t why_len,
                      int64_t *sizes, void *steps, int32_t *vars, float *fparams, void *wimg,
                      int32_t *root_map) {
    if (!valid_graph_handle(graph) || !is_layered || !sizes) return set_err(SPN_E_ARG, "bad arguments");
    LayeredPlan lp;
    detect_layered(*graph->graph, lp);
    *is_layered = lp.ok ? 1 : 0;
    if (why && why_len > 0) {
        strncpy(why, lp.why.c_str(), (size_t)why_len - 1);
        why[why_len - 1] = 0;
    }
    sizes[0] = (int64_t)lp.steps.size();
    sizes[1] = (int64_t)lp.vars.size();
    sizes[2] = (int64_t)lp.fparams.size();
    sizes[3] = (int64_t)lp.wimg.size() * 2;
    sizes[4] = (int64_t)lp.root_map.size();
    sizes[5] = lp.smem_floats;
    sizes[6] = (int64_t)sizeof(LStep);
    if (steps) memcpy(steps, lp.steps.data(), lp.steps.size() * sizeof(LStep));
    if (vars) memcpy(vars, lp.vars.data(), lp.vars.size() * 4);
    if (fparams) memcpy(fparams, lp.fparams.data(), lp.fparams.size() * 4);
    if (wimg) memcpy(wimg, lp.wimg.data(), lp.wimg.size() * 2);
    if (root_map) memcpy(root_map, lp.root_map.data(), lp.root_map.size() * 4);
    return SPN_OK;
}

int spn_codegen(const spn_handle *graph, int32_t task, int32_t lang, char *src, int64_t *src_len,
                char *name, int32_t *roots, int32_t *n_roots, float *tables, int64_t *n_tables,
                int32_t *n_tasks, int32_t compile, const char *arch) {
    if (!valid_graph_handle(graph) || !src_len || !n_roots || !n_tables || !n_tasks)
        return set_err(SPN_E_ARG, "bad arguments");
    JitOptions jo;
    if (const char *e = getenv("SPNB_JIT_K")) jo.samples_per_thread = std::min(4, std::max(1, atoi(e)));
    if (const char *e = getenv("SPNB_JIT_BAR")) jo.bar_every = std::max(0, atoi(e));
    if (const char *e = getenv("SPNB_JIT_MINB")) jo.min_blocks = std::max(1, atoi(e));
    // value space of the generated code: bits 8..9 of lang (0 auto, 1 log2, 2 linear)
    jo.space = (lang >> 8) & 3;
    lang &= 0xff;
    JitProgram jp;
    std::string msg;
    int rc = generate_jit(*graph->graph, jo, jp, msg);
    if (rc != SPN_OK) return set_err(rc, msg);
    *n_tasks = (int32_t)jp.tasks.size();
    if (task < 0 || task >= (int32_t)jp.tasks.size()) return set_err(SPN_E_ARG, "task out of range");
    const JitTask &t = jp.tasks[task];
    const std::string &text = lang == 1 ? t.source : t.cpp;
    if (src) {
        if (*src_len < (int64_t)text.size() + 1 || *n_roots < (int32_t)t.roots.size() ||
            *n_tables < (int64_t)jp.tables.size() || !roots || !tables)
            return set_err(SPN_E_ARG, "buffers too small");
        memcpy(src, text.c_str(), text.size() + 1);
        memcpy(roots, t.roots.data(), t.roots.size() * 4);
        memcpy(tables, jp.tables.data(), jp.tables.size() * 4);
        if (name) snprintf(name, 64, "%s", t.name.c_str());
    }
    *src_len = (int64_t)text.size() + 1;
    *n_roots = (int32_t)t.roots.size();
    *n_tables = (int64_t)jp.tables.size();
    if (compile) {
        std::vector<char> cubin;
        std::string log;
        for (int v = 0; v < 2; ++v) {
            rc = jit_compile(t.ptx[v], arch ? arch : "100a", cubin, log);
            if (rc != SPN_OK) return set_err(rc, log);
        }
    }
    return SPN_OK;
}

void spn_free(spn_handle *h) {
    if (!h) return;
    if (h->magic == H_GRAPH) delete h->graph;
    else if (h->magic == H_PLAN) free_plan(h->plan);
    h->magic = 0;
    delete h;
}

}  // extern "C"
