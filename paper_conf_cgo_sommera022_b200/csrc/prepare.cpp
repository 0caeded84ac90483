// prepare.cpp -- host-side graph preparer: validation, canonicalisation,
// ordering, acyclic partitioning into tasks, node-program generation with
// register-stack / slot allocation, and parameter packing.
//
// Paper correspondence (§IV-A):
//   * HiSPN canonicalisation: "transformation of DAG nodes with only a single
//     input" (L330)                                     -> canonicalise()
//   * graph partitioning (L336-346): initial partition from a depth-first
//     "ready" ordering (a node is appended once all its children are
//     processed), up to 1% balance slack, cost 1 per value crossing into a
//     partition (stored once, loaded once), Simple Moves refinement between
//     neighbouring partitions                           -> partition()
//   * bufferization / copy avoidance (L348-350): values crossing tasks go to
//     scratch slots allocated by liveness; task-local shared values to
//     shared-memory slots; outputs are written straight to the user buffer.
//   * the LoSPN body (L80-86): per task, a program over a register stack,
//     weighted sums lowered to max-shifted log-sum-exp in the log2 domain.
#include "prepare.h"

#include <algorithm>
#include <cmath>
#include <cstdio>
#include <cstring>
#include <functional>
#include <numeric>
#include <unordered_map>

#include "spnb.h"

namespace spnb {

namespace {

inline bool is_leaf(int32_t k) {
    return k == SPN_GAUSSIAN || k == SPN_CATEGORICAL || k == SPN_HISTOGRAM;
}

char g_buf[512];

int fail(std::string &msg, int code, const char *fmt, long long a = 0, long long b = 0) {
    snprintf(g_buf, sizeof(g_buf), fmt, a, b);
    msg = g_buf;
    return code;
}

inline uint32_t fbits(float f) {
    uint32_t u;
    memcpy(&u, &f, 4);
    return u;
}

}  // namespace

// ---------------------------------------------------------------------------
int validate_graph(const GraphData &g, std::string &msg) {
    const int64_t n = (int64_t)g.kind.size();
    const int64_t E = (int64_t)g.children.size();
    const int64_t P = (int64_t)g.params.size();
    if (g.F < 1) return fail(msg, SPN_E_ARG, "n_features must be >= 1");
    if (g.roots.empty()) return fail(msg, SPN_E_ARG, "need at least one root");
    for (int64_t u = 0; u < n; ++u) {
        const int32_t k = g.kind[u];
        if (k < 0 || k > 4) return fail(msg, SPN_E_GRAPH, "node %lld: bad kind %lld", u, k);
        if (is_leaf(k)) {
            if (g.n_children[u] != 0)
                return fail(msg, SPN_E_GRAPH, "leaf node %lld has children", u);
            if (g.feature[u] < 0 || g.feature[u] >= g.F)
                return fail(msg, SPN_E_GRAPH, "leaf node %lld: feature %lld out of range", u,
                            g.feature[u]);
            const int64_t pb = g.param_begin[u], np = g.n_params[u];
            if (pb < 0 || np < 0 || pb + np > P)
                return fail(msg, SPN_E_GRAPH, "leaf node %lld: params out of range", u);
            const double *p = g.params.data() + pb;
            if (k == SPN_GAUSSIAN) {
                if (np != 2) return fail(msg, SPN_E_GRAPH, "gaussian %lld: need 2 params", u);
                if (!std::isfinite(p[0]) || !std::isfinite(p[1]) || !(p[1] > 0.0))
                    return fail(msg, SPN_E_GRAPH, "gaussian %lld: bad mean/stddev", u);
            } else if (k == SPN_CATEGORICAL) {
                if (np < 1) return fail(msg, SPN_E_GRAPH, "categorical %lld: no probabilities", u);
                if (np > (1 << 22)) return fail(msg, SPN_E_UNSUPPORTED, "categorical %lld: too many categories", u);
                for (int64_t i = 0; i < np; ++i)
                    if (!(p[i] >= 0.0 && p[i] <= 1.0))
                        return fail(msg, SPN_E_GRAPH, "categorical %lld: probability %lld not in [0,1]", u, i);
            } else {
                if (np < 3 || np % 3 != 0)
                    return fail(msg, SPN_E_GRAPH, "histogram %lld: params must be (lb,ub,p) triples", u);
                std::vector<std::pair<double, double>> iv;
                double lo = INFINITY, hi = -INFINITY;
                for (int64_t b = 0; b < np; b += 3) {
                    const double lb = p[b], ub = p[b + 1], pr = p[b + 2];
                    if (!std::isfinite(lb) || !std::isfinite(ub) || lb != std::floor(lb) ||
                        ub != std::floor(ub) || !(lb < ub))
                        return fail(msg, SPN_E_GRAPH, "histogram %lld: bucket %lld needs integer lb < ub", u, b / 3);
                    if (!(pr >= 0.0 && pr <= 1.0))
                        return fail(msg, SPN_E_GRAPH, "histogram %lld: bucket %lld probability not in [0,1]", u, b / 3);
                    // fp32 inputs are exact integers only up to 2^24: the kernels compare
                    // x against the bounds in fp32 (larger bounds could
                    // index outside the table)
                    if (std::fabs(lb) > 16777216.0 || std::fabs(ub) > 16777216.0)
                        return fail(msg, SPN_E_UNSUPPORTED, "histogram %lld: bounds too large", u);
                    iv.push_back({lb, ub});
                    lo = std::min(lo, lb);
                    hi = std::max(hi, ub);
                }
                std::sort(iv.begin(), iv.end());
                for (size_t i = 1; i < iv.size(); ++i)
                    if (iv[i].first < iv[i - 1].second)
                        return fail(msg, SPN_E_GRAPH, "histogram %lld: overlapping buckets", u);
                if (hi - lo > (double)(1 << 22))
                    return fail(msg, SPN_E_UNSUPPORTED, "histogram %lld: range too wide for a table", u);
            }
        } else {
            const int64_t cb = g.child_begin[u], nc = g.n_children[u];
            if (nc < 1) return fail(msg, SPN_E_GRAPH, "inner node %lld has no children", u);
            if (cb < 0 || cb + nc > E)
                return fail(msg, SPN_E_GRAPH, "inner node %lld: children out of range", u);
            for (int64_t i = 0; i < nc; ++i) {
                const int64_t c = g.children[cb + i];
                if (c < 0 || c >= n)
                    return fail(msg, SPN_E_GRAPH, "node %lld: child index %lld out of range", u, c);
                if (k == SPN_SUM) {
                    const double w = g.weights[cb + i];
                    if (!(w >= 0.0) || !std::isfinite(w))
                        return fail(msg, SPN_E_GRAPH, "sum %lld: weight %lld negative/NaN/inf", u, i);
                }
            }
        }
    }
    for (size_t r = 0; r < g.roots.size(); ++r)
        if (g.roots[r] < 0 || g.roots[r] >= n)
            return fail(msg, SPN_E_GRAPH, "root %lld: node index %lld out of range", (long long)r,
                        g.roots[r]);
    // cycle check: iterative DFS, colours 0 white 1 grey 2 black
    std::vector<uint8_t> col(n, 0);
    std::vector<std::pair<int64_t, int64_t>> st;
    for (int64_t s = 0; s < n; ++s) {
        if (col[s]) continue;
        st.push_back({s, 0});
        col[s] = 1;
        while (!st.empty()) {
            auto &top = st.back();
            const int64_t u = top.first;
            const int64_t nc = is_leaf(g.kind[u]) ? 0 : g.n_children[u];
            if (top.second < nc) {
                const int64_t c = g.children[g.child_begin[u] + top.second++];
                if (col[c] == 1) return fail(msg, SPN_E_GRAPH, "cycle through node %lld", c);
                if (col[c] == 0) {
                    col[c] = 1;
                    st.push_back({c, 0});
                }
            } else {
                col[u] = 2;
                st.pop_back();
            }
        }
    }
    return SPN_OK;
}

// ---------------------------------------------------------------------------
namespace {

}  // namespace

void canonicalise(const GraphData &g, CGraph &c) {
    const int64_t n = (int64_t)g.kind.size();
    // rep(u): follow single-input nodes
    std::vector<int64_t> rep(n, -1);
    auto single = [&](int64_t u) -> bool {
        const int32_t k = g.kind[u];
        if (k == SPN_PRODUCT && g.n_children[u] == 1) return true;
        if (k == SPN_SUM && g.n_children[u] == 1 && g.weights[g.child_begin[u]] == 1.0) return true;
        return false;
    };
    for (int64_t u = 0; u < n; ++u) {
        if (rep[u] >= 0) continue;
        std::vector<int64_t> chain;
        int64_t v = u;
        while (rep[v] < 0 && single(v)) {
            chain.push_back(v);
            v = g.children[g.child_begin[v]];
        }
        const int64_t r = rep[v] >= 0 ? rep[v] : v;
        rep[v] = r;
        for (int64_t x : chain) rep[x] = r;
    }
    // post-order DFS from the roots over rep'd children
    std::vector<int64_t> newid(n, -1);
    std::vector<uint8_t> state(n, 0);
    std::vector<std::pair<int64_t, int64_t>> st;
    for (int64_t r0 : g.roots) {
        const int64_t r = rep[r0];
        if (state[r]) continue;
        st.push_back({r, 0});
        state[r] = 1;
        while (!st.empty()) {
            auto &top = st.back();
            const int64_t u = top.first;
            const int64_t nc = is_leaf(g.kind[u]) ? 0 : g.n_children[u];
            if (top.second < nc) {
                const int64_t cc = rep[g.children[g.child_begin[u] + top.second++]];
                if (!state[cc]) {
                    state[cc] = 1;
                    st.push_back({cc, 0});
                }
            } else {
                newid[u] = c.n++;
                c.orig.push_back(u);
                st.pop_back();
            }
        }
    }
    c.kind.resize(c.n);
    c.cb.assign(c.n + 1, 0);
    for (int64_t i = 0; i < c.n; ++i) {
        const int64_t u = c.orig[i];
        c.kind[i] = g.kind[u];
        c.cb[i + 1] = c.cb[i] + (is_leaf(g.kind[u]) ? 0 : g.n_children[u]);
    }
    c.ch.resize(c.cb[c.n]);
    c.w.resize(c.cb[c.n]);
    for (int64_t i = 0; i < c.n; ++i) {
        const int64_t u = c.orig[i];
        if (is_leaf(g.kind[u])) continue;
        for (int64_t j = 0; j < g.n_children[u]; ++j) {
            c.ch[c.cb[i] + j] = newid[rep[g.children[g.child_begin[u] + j]]];
            c.w[c.cb[i] + j] = g.kind[u] == SPN_SUM ? g.weights[g.child_begin[u] + j] : 0.0;
        }
    }
    // parents CSR
    std::vector<int64_t> cnt(c.n + 1, 0);
    for (int64_t e = 0; e < (int64_t)c.ch.size(); ++e) cnt[c.ch[e] + 1]++;
    c.pb.assign(c.n + 1, 0);
    for (int64_t i = 0; i < c.n; ++i) c.pb[i + 1] = c.pb[i] + cnt[i + 1];
    c.par.resize(c.ch.size());
    std::vector<int64_t> fill(c.pb.begin(), c.pb.end() - 1);
    for (int64_t i = 0; i < c.n; ++i)
        for (int64_t e = c.cb[i]; e < c.cb[i + 1]; ++e) c.par[fill[c.ch[e]]++] = i;
    c.rootrefs.assign(c.n, {});
    for (size_t r = 0; r < g.roots.size(); ++r) c.rootrefs[newid[rep[g.roots[r]]]].push_back((int32_t)r);
}

namespace {

// LoSPN-operation size of an inner node (binary mul/add after lowering,
// weighted sums become n muls + n-1 adds); leaf uses count 1.
int64_t op_size(const CGraph &c, int64_t u) {
    if (is_leaf(c.kind[u])) return 0;
    const int64_t n = c.cb[u + 1] - c.cb[u];
    int64_t leaves = 0;
    for (int64_t e = c.cb[u]; e < c.cb[u + 1]; ++e) leaves += is_leaf(c.kind[c.ch[e]]);
    return (c.kind[u] == SPN_SUM ? 2 * n - 1 : n - 1) + leaves;
}

// Number of distinct tasks other than task(v) that consume v, with node
// `moved` (a consumer) assumed to be in task `mt`.
int64_t value_cost(const CGraph &c, const std::vector<int32_t> &task, int64_t v, int64_t moved,
                   int32_t mt, int32_t tv, std::vector<int32_t> &scratch) {
    scratch.clear();
    for (int64_t e = c.pb[v]; e < c.pb[v + 1]; ++e) {
        const int64_t p = c.par[e];
        const int32_t tp = p == moved ? mt : task[p];
        if (tp != tv) scratch.push_back(tp);
    }
    std::sort(scratch.begin(), scratch.end());
    return (int64_t)(std::unique(scratch.begin(), scratch.end()) - scratch.begin());
}

PartitionResult partition(const CGraph &c, int64_t cap) {
    PartitionResult res;
    res.task.assign(c.n, -1);
    std::vector<int64_t> sz(c.n, 0);
    int64_t total = 0;
    for (int64_t u = 0; u < c.n; ++u) {
        sz[u] = op_size(c, u);
        total += sz[u];
    }
    if (cap <= 0 || total <= cap) {
        for (int64_t u = 0; u < c.n; ++u)
            if (!is_leaf(c.kind[u])) res.task[u] = 0;
        res.n_tasks = 1;
        return res;
    }
    // initial partition: chunks of the post-order ("ready" depth-first order,
    // L340) -- children precede parents, so chunks are acyclic.
    int32_t t = 0;
    int64_t cur = 0;
    std::vector<int64_t> tsize;
    tsize.push_back(0);
    for (int64_t u = 0; u < c.n; ++u) {
        if (is_leaf(c.kind[u])) continue;
        if (cur > 0 && cur + sz[u] > cap) {
            ++t;
            cur = 0;
            tsize.push_back(0);
        }
        res.task[u] = t;
        cur += sz[u];
        tsize[t] += sz[u];
    }
    int32_t T = t + 1;
    const int64_t slack_cap = (int64_t)std::ceil(1.01 * (double)cap);  // 1% slack (L342)
    // Simple Moves refinement between neighbouring partitions (L346, reading c14)
    std::vector<int32_t> scratch;
    std::vector<int64_t> kids;
    for (int pass = 0; pass < 8; ++pass) {
        int64_t moves = 0;
        for (int64_t u = 0; u < c.n; ++u) {
            if (is_leaf(c.kind[u])) continue;
            const int32_t k = res.task[u];
            kids.clear();
            for (int64_t e = c.cb[u]; e < c.cb[u + 1]; ++e)
                if (!is_leaf(c.kind[c.ch[e]])) kids.push_back(c.ch[e]);
            std::sort(kids.begin(), kids.end());
            kids.erase(std::unique(kids.begin(), kids.end()), kids.end());
            for (int dir = -1; dir <= 1; dir += 2) {
                const int32_t tt = k + dir;
                if (tt < 0 || tt >= T) continue;
                if (tsize[tt] + sz[u] > slack_cap) continue;
                bool ok = true;
                if (dir < 0) {
                    for (int64_t cc : kids)
                        if (res.task[cc] > tt) { ok = false; break; }
                } else {
                    for (int64_t e = c.pb[u]; e < c.pb[u + 1]; ++e)
                        if (res.task[c.par[e]] < tt) { ok = false; break; }
                }
                if (!ok) continue;
                int64_t before = value_cost(c, res.task, u, -1, 0, k, scratch);
                int64_t after = value_cost(c, res.task, u, -1, 0, tt, scratch);
                for (int64_t cc : kids) {
                    before += value_cost(c, res.task, cc, -1, 0, res.task[cc], scratch);
                    after += value_cost(c, res.task, cc, u, tt, res.task[cc], scratch);
                }
                if (after < before) {
                    res.task[u] = tt;
                    tsize[k] -= sz[u];
                    tsize[tt] += sz[u];
                    ++moves;
                    break;
                }
            }
        }
        if (!moves) break;
    }
    // drop empty tasks
    std::vector<int32_t> remap(T, -1);
    int32_t nt = 0;
    for (int32_t i = 0; i < T; ++i)
        if (tsize[i] > 0) remap[i] = nt++;
    for (int64_t u = 0; u < c.n; ++u)
        if (res.task[u] >= 0) res.task[u] = remap[res.task[u]];
    res.n_tasks = nt;
    for (int64_t u = 0; u < c.n; ++u) {
        if (is_leaf(c.kind[u])) continue;
        const int64_t vc = value_cost(c, res.task, u, -1, 0, res.task[u], scratch);
        res.cost += vc;
        res.cut_values += vc > 0;
    }
    return res;
}

// Pack a leaf's parameters.
struct LeafPack {
    bool gauss;    // Gaussian (else discrete table)
    uint32_t f;    // feature
    uint32_t y, z, w;
    double c;      // Gaussian: -log2(sigma sqrt(2 pi)) (pre-summed into LPUSH's C)
};

}  // namespace

// ---------------------------------------------------------------------------
int build_program(const GraphData &g, const CodegenConfig &cfg, PlanProgram &out,
                  std::string &msg) {
    CGraph c;
    canonicalise(g, c);
    const int K = cfg.K;
    const int WT = 32 * K;
    out.n_nodes = c.n;
    out.n_roots = (int64_t)g.roots.size();

    // ---- statistics (algorithmic counts on the canonical graph) ----
    for (int64_t u = 0; u < c.n; ++u) {
        const int64_t nc = c.cb[u + 1] - c.cb[u];
        if (is_leaf(c.kind[u])) {
            out.n_leaves++;
            out.fma_per_sample += 2;
        } else if (c.kind[u] == SPN_SUM) {
            out.n_sums++;
            out.n_sum_edges += nc;
            out.mufu_per_sample += nc > 1 ? nc : 0;  // n-ary LSE: n-1 ex2 + 1 lg2
            out.fma_per_sample += 3 * nc;
        } else {
            out.n_products++;
            out.fma_per_sample += nc - 1;
        }
    }

    // ---- leaf packing (log2 domain) ----
    std::vector<LeafPack> leaf(c.n);
    for (int64_t u = 0; u < c.n; ++u) {
        const int64_t o = c.orig[u];
        if (!is_leaf(c.kind[u])) continue;
        LeafPack lp;
        lp.f = (uint32_t)g.feature[o];
        const double *p = g.params.data() + g.param_begin[o];
        const int64_t np = g.n_params[o];
        if (c.kind[u] == SPN_GAUSSIAN) {
            const double mu = p[0], sd = p[1];
            const double a = 1.0 / (sd * std::sqrt(2.0 * M_LN2));
            const double b = a * mu;
            const double cc = -std::log2(sd * std::sqrt(2.0 * M_PI));
            lp.gauss = true;
            lp.c = cc;
            lp.y = fbits((float)a);
            lp.z = fbits((float)b);
            lp.w = fbits((float)cc);
        } else {
            int64_t lo, nk;
            std::vector<float> tab;
            if (c.kind[u] == SPN_CATEGORICAL) {
                lo = 0;
                nk = np;
                tab.resize(nk);
                for (int64_t i = 0; i < nk; ++i) tab[i] = (float)std::log2(p[i]);
            } else {
                double mn = INFINITY, mx = -INFINITY;
                for (int64_t b = 0; b < np; b += 3) {
                    mn = std::min(mn, p[b]);
                    mx = std::max(mx, p[b + 1]);
                }
                lo = (int64_t)mn;
                nk = (int64_t)mx - lo;
                tab.assign(nk, -INFINITY);
                for (int64_t b = 0; b < np; b += 3)
                    for (int64_t v = (int64_t)p[b]; v < (int64_t)p[b + 1]; ++v)
                        tab[v - lo] = (float)std::log2(p[b + 2]);
            }
            lp.gauss = false;
            lp.c = 0.0;
            lp.y = (uint32_t)out.tables.size();
            lp.z = (uint32_t)(int32_t)lo;
            lp.w = (uint32_t)nk;
            out.tables.insert(out.tables.end(), tab.begin(), tab.end());
        }
        leaf[u] = lp;
    }
    if (out.tables.empty()) out.tables.push_back(0.f);

    // ---- partitioning ----
    PartitionResult part = partition(c, cfg.max_task_ops);
    const int32_t T = part.n_tasks;
    out.n_cut_values = part.cut_values;
    out.partition_cost = part.cost;
    auto task_of = [&](int64_t u) -> int32_t { return is_leaf(c.kind[u]) ? 0 : part.task[u]; };

    // ---- materialisation decisions ----
    std::vector<uint8_t> mat(c.n, 0), virt(c.n, 0), glse(c.n, 0), cross(c.n, 0);
    for (int64_t u = 0; u < c.n; ++u) {
        if (is_leaf(c.kind[u])) continue;  // leaves are rematerialised at each use
        const int64_t cons = c.pb[u + 1] - c.pb[u];
        const int64_t nr = (int64_t)c.rootrefs[u].size();
        for (int64_t e = c.pb[u]; e < c.pb[u + 1]; ++e)
            if (part.task[c.par[e]] != part.task[u]) cross[u] = 1;
        if (cons + nr > 1 || cross[u]) mat[u] = 1;
    }
    auto fan = [&](int64_t u) { return c.cb[u + 1] - c.cb[u]; };
    // candidate virtual products: two stored inner children, consumed only by
    // large sums of the same task (gather-LSE terms slot(a) + slot(b)).
    std::vector<uint8_t> vcand(c.n, 0);
    for (int64_t u = 0; u < c.n; ++u) {
        if (c.kind[u] != SPN_PRODUCT || !mat[u] || cross[u] || !c.rootrefs[u].empty()) continue;
        if (fan(u) != 2) continue;
        const int64_t a = c.ch[c.cb[u]], b = c.ch[c.cb[u] + 1];
        if (is_leaf(c.kind[a]) || is_leaf(c.kind[b]) || !mat[a] || !mat[b]) continue;
        bool ok = true;
        for (int64_t e = c.pb[u]; e < c.pb[u + 1]; ++e) {
            const int64_t p = c.par[e];
            if (c.kind[p] != SPN_SUM || fan(p) <= cfg.lse_max) { ok = false; break; }
        }
        vcand[u] = ok;
    }
    for (int64_t u = 0; u < c.n; ++u) {
        if (c.kind[u] != SPN_SUM || fan(u) <= cfg.lse_max) continue;
        bool ok = true;
        for (int64_t e = c.cb[u]; e < c.cb[u + 1]; ++e) {
            const int64_t ch = c.ch[e];
            if (is_leaf(c.kind[ch]) || !(mat[ch] || vcand[ch])) { ok = false; break; }
        }
        glse[u] = ok;
    }
    for (int64_t u = 0; u < c.n; ++u) {
        if (!vcand[u]) continue;
        bool ok = true;
        for (int64_t e = c.pb[u]; e < c.pb[u + 1]; ++e)
            if (!glse[c.par[e]]) { ok = false; break; }
        if (ok) {
            virt[u] = 1;
            mat[u] = 0;
        }
    }

    // ---- Sethi-Ullman stack needs; force-materialise subtrees that would
    //      overflow the MAXD-deep register stack ----
    std::vector<int32_t> need(c.n, 1);
    std::vector<int64_t> order_buf;
    auto child_need = [&](int64_t ch) -> int32_t {
        if (is_leaf(c.kind[ch]) || mat[ch]) return 1;
        return need[ch];
    };
    // fused sum of Gaussian leaf products (SLPk): 2..4 children, each a
    // Gaussian leaf or an unshared product of 1..7 Gaussian leaves
    auto gprod_leaves = [&](int64_t ch) -> int {
        if (c.kind[ch] == SPN_GAUSSIAN) return 1;
        if (c.kind[ch] != SPN_PRODUCT || mat[ch] || virt[ch]) return 0;
        int cnt = 0;
        for (int64_t e = c.cb[ch]; e < c.cb[ch + 1]; ++e) {
            if (c.kind[c.ch[e]] != SPN_GAUSSIAN) return 0;
            ++cnt;
        }
        return cnt <= 7 ? cnt : 0;
    };
    auto slp_ok = [&](int64_t u) -> bool {
        if (c.kind[u] != SPN_SUM || glse[u]) return false;
        const int64_t n = fan(u);
        if (n < 2 || n > 4) return false;
        for (int64_t e = c.cb[u]; e < c.cb[u + 1]; ++e)
            if (!gprod_leaves(c.ch[e])) return false;
        return true;
    };
    auto compute_need = [&](int64_t u) -> int32_t {
        const int32_t k = c.kind[u];
        if (is_leaf(k) || virt[u]) return 1;
        if (k == SPN_SUM && (glse[u] || slp_ok(u))) return 1;
        std::vector<int32_t> nv;
        int nleaf = 0;
        for (int64_t e = c.cb[u]; e < c.cb[u + 1]; ++e) {
            const int64_t ch = c.ch[e];
            if (k == SPN_PRODUCT && is_leaf(c.kind[ch])) {
                ++nleaf;
                continue;
            }
            nv.push_back(child_need(ch));
        }
        std::sort(nv.rbegin(), nv.rend());
        int32_t r = 1;
        if (k == SPN_PRODUCT) {
            for (size_t i = 0; i < nv.size(); ++i) r = std::max(r, nv[i] + (i > 0 ? 1 : 0));
            if (nv.empty()) r = 1;
        } else {
            const int n = (int)nv.size();
            if (n <= cfg.lse_max) {
                for (int i = 0; i < n; ++i) r = std::max(r, nv[i] + i);
            } else {
                for (int i = 0; i < 4 && i < n; ++i) r = std::max(r, nv[i] + i);
                for (int i = 4; i < n; ++i) r = std::max(r, nv[i] + 1 + (i - 4) % 3);
            }
        }
        return r;
    };
    for (int64_t u = 0; u < c.n; ++u) {
        if (is_leaf(c.kind[u])) continue;
        int32_t nd = compute_need(u);
        while (nd > cfg.maxd) {
            // materialise the non-stored inner child with the largest need
            int64_t best = -1;
            int32_t bn = 0;
            for (int64_t e = c.cb[u]; e < c.cb[u + 1]; ++e) {
                const int64_t ch = c.ch[e];
                if (is_leaf(c.kind[ch]) || mat[ch] || virt[ch]) continue;
                if (need[ch] > bn) {
                    bn = need[ch];
                    best = ch;
                }
            }
            if (best < 0) return fail(msg, SPN_E_UNSUPPORTED, "node %lld: stack need %lld exceeds the register stack", u, nd);
            mat[best] = 1;
            nd = compute_need(u);
        }
        need[u] = nd;
    }

    // ---- code generation ----
    // emit_value(u, sp, bias) leaves value(u) + bias at stack position sp.
    // bias carries the parent sum's log2 weight (weights are folded into the
    // records producing the children, so LSE records need no weight adds).
    struct Fix {
        int64_t idx;      // record index or edge index
        int64_t node;
        int kind;         // 0 load rec, 1 store rec, 2 edge.a, 3 edge.b
    };
    std::vector<Fix> fixes;
    std::vector<Rec> &prog = out.prog;
    int64_t max_sp = 0;
    bool overflow = false;
    auto rec_of = [&](uint32_t op, int sp, uint32_t arg, uint32_t y = 0, uint32_t z = 0,
                      uint32_t w = 0) {
        if (sp > cfg.maxd || sp < 0 || arg > ARG_MAX) {
            overflow = true;
            return;
        }
        prog.push_back(make_rec(op, (uint32_t)sp, arg, y, z, w));
    };
    auto feat_arg = [&](uint32_t f) -> uint32_t {
        return cfg.x_in_smem ? f * (uint32_t)cfg.tpw * 4u : f * 4u;
    };
    auto lw2 = [](double w) -> double { return std::log2(w); };
    // leaf product: LPUSH (acc=false, pushes at sp) or LACC (adds to r[sp])
    auto emit_leaves = [&](const std::vector<int64_t> &lv, int sp, bool acc, double bias) {
        double C = bias;
        uint32_t ng = 0, nd = 0;
        for (int64_t u : lv) {
            if (leaf[u].gauss) {
                C += leaf[u].c;
                ++ng;
            } else {
                ++nd;
            }
        }
        if (!acc) max_sp = std::max<int64_t>(max_sp, sp + 1);
        bool packable = nd == 0 && ng >= 1 && ng <= 4;
        uint32_t fo[4] = {0, 0, 0, 0};
        if (packable) {
            int k = 0;
            for (int64_t u : lv) {
                const uint32_t f = feat_arg(leaf[u].f);
                if (f > 0xffffu) packable = false;
                fo[k++] = f;
            }
        }
        if (packable)  // straight-line variants, feature offsets in the header
            rec_of((acc ? OP_GACC1 : OP_GPUSH1) + ng - 1, acc ? sp + 1 : sp, 0, fbits((float)C),
                   fo[0] | (fo[1] << 16), fo[2] | (fo[3] << 16));
        else
            rec_of(acc ? OP_LACC : OP_LPUSH, acc ? sp + 1 : sp, ng, fbits((float)C), nd);
        for (int pass = 0; pass < 2; ++pass)
            for (int64_t u : lv) {
                const LeafPack &lp = leaf[u];
                if (lp.gauss != (pass == 0)) continue;
                prog.push_back(Rec{feat_arg(lp.f), lp.y, lp.z, lp.w});
            }
    };
    auto emit_load = [&](int64_t u, int sp, double bias) {
        max_sp = std::max<int64_t>(max_sp, sp + 1);
        fixes.push_back({(int64_t)prog.size(), u, 0});
        rec_of(OP_LDS, sp, 0, fbits((float)bias));
    };
    std::function<void(int64_t, int, double)> emit_value;
    auto emit_child = [&](int64_t ch, int sp, double bias) {
        if (!is_leaf(c.kind[ch]) && mat[ch]) emit_load(ch, sp, bias);
        else emit_value(ch, sp, bias);
    };
    emit_value = [&](int64_t u, int sp, double bias) {
        const int32_t k = c.kind[u];
        if (is_leaf(k)) {
            emit_leaves({u}, sp, false, bias);
            return;
        }
        if (k == SPN_PRODUCT) {
            std::vector<std::pair<int32_t, int64_t>> inner;
            std::vector<int64_t> leaves;
            for (int64_t e = c.cb[u]; e < c.cb[u + 1]; ++e) {
                const int64_t ch = c.ch[e];
                if (is_leaf(c.kind[ch])) leaves.push_back(ch);
                else inner.push_back({child_need(ch), ch});
            }
            std::stable_sort(inner.begin(), inner.end(),
                             [](auto &a, auto &b) { return a.first > b.first; });
            if (inner.empty()) {
                emit_leaves(leaves, sp, false, bias);
                return;
            }
            for (size_t i = 0; i < inner.size(); ++i) {
                const bool last_add = leaves.empty() && i + 1 == inner.size();
                if (i == 0) {
                    emit_child(inner[i].second, sp, inner.size() == 1 && leaves.empty() ? bias : 0.0);
                } else {
                    emit_child(inner[i].second, sp + 1, 0.0);
                    rec_of(OP_ADD, sp + 2, 0, fbits((float)(last_add ? bias : 0.0)));
                }
            }
            if (!leaves.empty()) emit_leaves(leaves, sp, true, bias);
            return;
        }
        // weighted sum
        const int64_t n = fan(u);
        if (n == 1) {  // single-input sum with weight != 1: value + log2 w
            emit_child(c.ch[c.cb[u]], sp, bias + lw2(c.w[c.cb[u]]));
            return;
        }
        if (glse[u]) {
            const int64_t off = (int64_t)out.edges.size();
            for (int64_t e = c.cb[u]; e < c.cb[u + 1]; ++e) {
                const int64_t ch = c.ch[e];
                Edge ed;
                ed.lw = (float)(lw2(c.w[e]) + bias);
                ed.pad = 0;
                ed.a = 0;
                ed.b = SLOT_NONE;
                const int64_t ei = (int64_t)out.edges.size();
                if (virt[ch]) {
                    fixes.push_back({ei, c.ch[c.cb[ch]], 2});
                    fixes.push_back({ei, c.ch[c.cb[ch] + 1], 3});
                } else {
                    fixes.push_back({ei, ch, 2});
                }
                out.edges.push_back(ed);
            }
            max_sp = std::max<int64_t>(max_sp, sp + 1);
            rec_of(OP_GLSE, sp, 0, (uint32_t)(off & 0xffffffffu), (uint32_t)(off >> 32), (uint32_t)n);
            return;
        }
        if (slp_ok(u)) {
            uint32_t counts = 0, Cb[4] = {0, 0, 0, 0};
            std::vector<int64_t> lv;
            for (int64_t e = c.cb[u], ci = 0; e < c.cb[u + 1]; ++e, ++ci) {
                const int64_t ch = c.ch[e];
                std::vector<int64_t> cl;
                if (c.kind[ch] == SPN_GAUSSIAN) cl.push_back(ch);
                else cl.assign(c.ch.begin() + c.cb[ch], c.ch.begin() + c.cb[ch + 1]);
                double C = lw2(c.w[e]);
                for (int64_t l : cl) C += leaf[l].c;
                Cb[ci] = fbits((float)C);
                counts |= (uint32_t)cl.size() << (3 * ci);
                lv.insert(lv.end(), cl.begin(), cl.end());
            }
            max_sp = std::max<int64_t>(max_sp, sp + 1);
            // straight-line form for children of exactly 2 leaves (n = 2, 3)
            bool uni = (n == 2 || n == 3) && counts == (n == 2 ? 0x12u : 0x92u);
            uint32_t fo[6] = {0, 0, 0, 0, 0, 0};
            if (uni) {
                for (size_t k = 0; k < lv.size(); ++k) {
                    fo[k] = feat_arg(leaf[lv[k]].f);
                    if (fo[k] > 0xffffu) uni = false;
                }
            }
            if (uni && n == 2) {
                rec_of(OP_SLPU2, sp, 0, fbits((float)bias), Cb[0], Cb[1]);
                prog.push_back(Rec{fo[0] | (fo[1] << 16), fo[2] | (fo[3] << 16), 0, 0});
            } else if (uni) {
                rec_of(OP_SLPU3, sp, 0, fbits((float)bias), Cb[0], Cb[1]);
                prog.push_back(Rec{Cb[2], fo[0] | (fo[1] << 16), fo[2] | (fo[3] << 16),
                                   fo[4] | (fo[5] << 16)});
            } else {
                rec_of(OP_SLP2 + (uint32_t)(n - 2), sp, counts, fbits((float)bias), Cb[0], Cb[1]);
                if (n >= 3) prog.push_back(Rec{Cb[2], Cb[3], 0, 0});
            }
            for (int64_t l : lv) prog.push_back(Rec{feat_arg(leaf[l].f), leaf[l].y, leaf[l].z, leaf[l].w});
            return;
        }
        std::vector<std::pair<int32_t, int64_t>> kids;  // (need, edge)
        for (int64_t e = c.cb[u]; e < c.cb[u + 1]; ++e) kids.push_back({child_need(c.ch[e]), e});
        std::stable_sort(kids.begin(), kids.end(),
                         [](auto &a, auto &b) { return a.first > b.first; });
        if (n <= cfg.lse_max) {
            for (int64_t i = 0; i < n; ++i)
                emit_child(c.ch[kids[i].second], sp + (int)i, lw2(c.w[kids[i].second]));
            rec_of(OP_LSE1 + (uint32_t)(n - 1), sp + (int)n, 0, fbits((float)bias));
            return;
        }
        // chunked: first 4 children, then (accumulator + up to 3 children)
        for (int i = 0; i < 4; ++i)
            emit_child(c.ch[kids[i].second], sp + i, lw2(c.w[kids[i].second]));
        rec_of(OP_LSE4, sp + 4, 0, fbits(n == 4 ? (float)bias : 0.f));
        for (int64_t i = 4; i < n; i += 3) {
            const int64_t m = std::min<int64_t>(3, n - i);
            for (int64_t j = 0; j < m; ++j)
                emit_child(c.ch[kids[i + j].second], sp + 1 + (int)j, lw2(c.w[kids[i + j].second]));
            const bool last = i + m >= n;
            rec_of(OP_LSE1 + (uint32_t)m, sp + 1 + (int)m, 0, fbits(last ? (float)bias : 0.f));
        }
    };

    std::vector<int64_t> store_rec(c.n, -1);
    out.task_off.clear();
    std::vector<std::vector<int64_t>> task_nodes(T);
    for (int64_t u = 0; u < c.n; ++u) task_nodes[task_of(u)].push_back(u);
    for (int32_t t = 0; t < T; ++t) {
        out.task_off.push_back((int64_t)prog.size());
        for (int64_t u : task_nodes[t]) {
            const bool is_root = !c.rootrefs[u].empty();
            if (is_leaf(c.kind[u])) {
                if (!is_root) continue;
                emit_leaves({u}, 0, false, 0.0);
            } else {
                if (virt[u]) continue;
                if (!mat[u] && !is_root) continue;  // emitted inside its consumer
                emit_value(u, 0, 0.0);
                if (mat[u]) {
                    store_rec[u] = (int64_t)prog.size();
                    fixes.push_back({(int64_t)prog.size(), u, 1});
                    rec_of(OP_STS, 1, 0);
                }
            }
            for (int32_t r : c.rootrefs[u]) rec_of(OP_OUT, 1, (uint32_t)r);
        }
        prog.push_back(make_rec(OP_END, 0, 0));
    }
    out.task_off.push_back((int64_t)prog.size());
    if (overflow || max_sp > cfg.maxd)
        return fail(msg, SPN_E_UNSUPPORTED, "register stack overflow (depth %lld)", max_sp);
    out.max_stack = max_sp;
    for (int32_t t = 0; t < T; ++t)
        out.max_task_records = std::max(out.max_task_records, out.task_off[t + 1] - out.task_off[t]);

    // ---- slot allocation by liveness (linear scan over record order) ----
    std::vector<int64_t> last_use(c.n, -1);
    // edge fixups belong to the GLSE record that owns them: map edge -> record
    std::vector<int64_t> edge_rec(out.edges.size(), -1);
    for (int64_t i = 0; i < (int64_t)prog.size(); ++i) {
        const uint32_t cs = prog[i].x & ((1u << CASE_BITS) - 1u);
        if (cs / NSP == OP_GLSE && cs < OP_COUNT * NSP) {
            const int64_t off = ((int64_t)prog[i].z << 32) | prog[i].y;
            for (int64_t e = off; e < off + (int64_t)prog[i].w; ++e) edge_rec[e] = i;
        }
        if ((cs / NSP == OP_LPUSH || cs / NSP == OP_LACC) && cs < OP_COUNT * NSP)
            i += (int64_t)(prog[i].x >> CASE_BITS) + (int64_t)prog[i].z;  // skip leaf params
        else if (cs / NSP >= OP_GPUSH1 && cs / NSP <= OP_GPUSH4)
            i += cs / NSP - OP_GPUSH1 + 1;
        else if (cs / NSP >= OP_GACC1 && cs / NSP <= OP_GACC4)
            i += cs / NSP - OP_GACC1 + 1;
        else if (cs / NSP == OP_SLPU2 && cs < OP_COUNT * NSP)
            i += 1 + 4;
        else if (cs / NSP == OP_SLPU3 && cs < OP_COUNT * NSP)
            i += 1 + 6;
        else if (cs / NSP >= OP_SLP2 && cs / NSP <= OP_SLP4 && cs < OP_COUNT * NSP) {
            const uint32_t cnt = prog[i].x >> CASE_BITS;
            i += (cs / NSP >= OP_SLP3 ? 1 : 0) + (cnt & 7u) + ((cnt >> 3) & 7u) +
                 ((cnt >> 6) & 7u) + ((cnt >> 9) & 7u);
        }
    }
    for (const Fix &f : fixes) {
        if (f.kind == 0) last_use[f.node] = std::max(last_use[f.node], f.idx);
        else if (f.kind >= 2) last_use[f.node] = std::max(last_use[f.node], edge_rec[f.idx]);
    }
    std::vector<int64_t> slot_of(c.n, -1);
    std::vector<uint8_t> in_global(c.n, 0);
    std::vector<std::vector<int64_t>> frees(prog.size() + 1);
    for (int64_t u = 0; u < c.n; ++u)
        if (store_rec[u] >= 0) frees[std::max(last_use[u], store_rec[u])].push_back(u);
    std::vector<int64_t> free_s, free_g;
    int64_t n_s = 0, n_g = 0;
    std::vector<int64_t> store_at(prog.size(), -1);
    for (int64_t u = 0; u < c.n; ++u)
        if (store_rec[u] >= 0) store_at[store_rec[u]] = u;
    for (int64_t i = 0; i < (int64_t)prog.size(); ++i) {
        const int64_t u = store_at[i];
        if (u >= 0) {
            const bool glob = cross[u] != 0;
            if (!glob && (!free_s.empty() || n_s < cfg.smem_slot_cap)) {
                if (!free_s.empty()) {
                    slot_of[u] = free_s.back();
                    free_s.pop_back();
                } else {
                    slot_of[u] = n_s++;
                }
            } else {
                in_global[u] = 1;
                if (!free_g.empty()) {
                    slot_of[u] = free_g.back();
                    free_g.pop_back();
                } else {
                    slot_of[u] = n_g++;
                }
            }
        }
        for (int64_t v : frees[i]) {
            if (slot_of[v] < 0) continue;
            if (in_global[v]) free_g.push_back(slot_of[v]);
            else free_s.push_back(slot_of[v]);
        }
    }
    out.n_sslots = n_s;
    out.n_gslots = n_g;
    const uint64_t slot_bytes = (uint64_t)WT * 4u;
    for (const Fix &f : fixes) {
        const int64_t u = f.node;
        if (slot_of[u] < 0) return fail(msg, SPN_E_UNSUPPORTED, "internal: node %lld has no slot", u);
        const uint64_t off = (uint64_t)slot_of[u] * slot_bytes;
        // shared slots: byte offset in the 23-bit record argument; global
        // slots: in the record's z word / the edge ref (31 bits)
        if ((!in_global[u] && off > ARG_MAX) || off >= SLOT_GLOBAL)
            return fail(msg, SPN_E_UNSUPPORTED, "too many scratch slots (%lld)", slot_of[u]);
        if (f.kind <= 1) {
            Rec &r = prog[f.idx];
            const uint32_t sp = (r.x & ((1u << CASE_BITS) - 1u)) % NSP;
            uint32_t op;
            if (f.kind == 0) op = in_global[u] ? OP_LDG : OP_LDS;
            else op = in_global[u] ? OP_STG : OP_STS;
            if (in_global[u]) r = make_rec(op, sp, 0u, r.y, (uint32_t)off, r.w);
            else r = make_rec(op, sp, (uint32_t)off, r.y, r.z, r.w);
        } else {
            const uint32_t ref = (uint32_t)off | (in_global[u] ? SLOT_GLOBAL : 0u);
            if (f.kind == 2) out.edges[f.idx].a = ref;
            else out.edges[f.idx].b = ref;
        }
    }
    if (out.edges.empty()) out.edges.push_back(Edge{0, SLOT_NONE, 0.f, 0});
    return SPN_OK;
}

// Partition only (host introspection for tests): task per ORIGINAL node.
int partition_graph(const GraphData &g, int64_t cap, std::vector<int32_t> &task_of_orig,
                    PartitionResult &res) {
    CGraph c;
    canonicalise(g, c);
    res = partition(c, cap);
    task_of_orig.assign(g.kind.size(), -1);
    for (int64_t u = 0; u < c.n; ++u)
        if (!is_leaf(c.kind[u])) task_of_orig[c.orig[u]] = res.task[u];
    return SPN_OK;
}

}  // namespace spnb
