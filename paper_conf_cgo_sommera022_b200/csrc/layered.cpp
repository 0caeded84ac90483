// layered.cpp -- detection of RAT-SPN-style region graphs and construction of
// the tensor-core plan (see layered.h, rat_eval.cu).
#include "layered.h"

#include <algorithm>
#include <cmath>
#include <cstring>
#include <functional>
#include <map>
#include <unordered_map>

#include "spnb.h"

namespace spnb {

namespace {

inline bool is_leafk(int32_t k) {
    return k == SPN_GAUSSIAN || k == SPN_CATEGORICAL || k == SPN_HISTOGRAM;
}

uint16_t f32_to_f16(float f) {
    // round-to-nearest-even conversion (host)
    uint32_t x;
    memcpy(&x, &f, 4);
    const uint32_t sign = (x >> 16) & 0x8000u;
    int32_t exp = (int32_t)((x >> 23) & 0xff) - 127 + 15;
    uint32_t man = x & 0x7fffffu;
    if (((x >> 23) & 0xff) == 0xff) return (uint16_t)(sign | 0x7c00u | (man ? 0x200u : 0));
    if (exp >= 31) return (uint16_t)(sign | 0x7c00u);
    if (exp <= 0) {
        if (exp < -10) return (uint16_t)sign;
        man |= 0x800000u;
        const int shift = 14 - exp;
        uint32_t h = man >> shift;
        const uint32_t rem = man & ((1u << shift) - 1);
        const uint32_t half = 1u << (shift - 1);
        if (rem > half || (rem == half && (h & 1))) ++h;
        return (uint16_t)(sign | h);
    }
    uint32_t h = ((uint32_t)exp << 10) | (man >> 13);
    const uint32_t rem = man & 0x1fffu;
    if (rem > 0x1000u || (rem == 0x1000u && (h & 1))) ++h;
    return (uint16_t)(sign | h);
}

float f16_to_f32(uint16_t h) {
    const uint32_t sign = (uint32_t)(h & 0x8000u) << 16;
    uint32_t exp = (h >> 10) & 0x1f, man = h & 0x3ffu;
    uint32_t x;
    if (exp == 0) {
        if (man == 0) {
            x = sign;
        } else {
            int e = -1;
            do {
                ++e;
                man <<= 1;
            } while (!(man & 0x400u));
            x = sign | ((uint32_t)(127 - 15 - e) << 23) | ((man & 0x3ffu) << 13);
        }
    } else if (exp == 31) {
        x = sign | 0x7f800000u | (man << 13);
    } else {
        x = sign | ((exp - 15 + 127) << 23) | (man << 13);
    }
    float f;
    memcpy(&f, &x, 4);
    return f;
}

uint64_t hash_vec(const std::vector<int64_t> &v) {
    uint64_t h = 1469598103934665603ull;
    for (int64_t x : v) {
        h ^= (uint64_t)x + 0x9e3779b97f4a7c15ull + (h << 6) + (h >> 2);
        h *= 1099511628211ull;
    }
    return h;
}

struct Region {
    bool leaf = false;
    std::vector<int64_t> nodes;          // value index -> canonical node
    std::vector<int32_t> vars;           // leaf regions: sorted features
    std::vector<int32_t> partitions;     // sum regions: partitions feeding the sums
    int32_t consumer_partition = -1;
};

struct Partition {
    int32_t ra = -1, rb = -1;            // child regions (ra < rb)
    std::vector<int64_t> prods;          // cell (i*nb + j) -> product node
    int32_t consumer_region = -1;
};

}  // namespace

void detect_layered(const GraphData &g, LayeredPlan &plan, int n_cap) {
    plan = LayeredPlan();
    CGraph c;
    canonicalise(g, c);
    auto fail = [&](const std::string &why) {
        plan.ok = false;
        plan.why = why;
    };
    auto fan = [&](int64_t u) { return c.cb[u + 1] - c.cb[u]; };
    const int64_t n = c.n;
    std::vector<int32_t> region_of(n, -1), index_in(n, -1);
    std::vector<Region> regions;

    // ---- leaf regions: Gaussian leaves / products of Gaussian leaves over
    //      distinct variables, grouped by variable set
    std::map<std::vector<int32_t>, int32_t> by_vars;
    std::vector<int32_t> feats;
    for (int64_t u = 0; u < n; ++u) {
        feats.clear();
        if (c.kind[u] == SPN_GAUSSIAN) {
            // a Gaussian consumed by anything but products of leaves is a 1-var dist
            bool in_leaf_product = c.pb[u + 1] > c.pb[u];
            for (int64_t e = c.pb[u]; e < c.pb[u + 1]; ++e) {
                const int64_t p = c.par[e];
                bool all_g = c.kind[p] == SPN_PRODUCT;
                for (int64_t f = c.cb[p]; all_g && f < c.cb[p + 1]; ++f)
                    all_g = c.kind[c.ch[f]] == SPN_GAUSSIAN;
                if (!all_g) in_leaf_product = false;
            }
            if (in_leaf_product) continue;  // part of a factorised distribution
            feats.push_back(g.feature[c.orig[u]]);
        } else if (c.kind[u] == SPN_PRODUCT) {
            bool all_g = true;
            for (int64_t e = c.cb[u]; e < c.cb[u + 1] && all_g; ++e) {
                const int64_t ch = c.ch[e];
                all_g = c.kind[ch] == SPN_GAUSSIAN;
                if (all_g) feats.push_back(g.feature[c.orig[ch]]);
            }
            if (!all_g) continue;
            std::sort(feats.begin(), feats.end());
            if (std::adjacent_find(feats.begin(), feats.end()) != feats.end())
                return fail("leaf product repeats a variable");
        } else {
            if (is_leafk(c.kind[u])) return fail("discrete leaves are not layered");
            continue;
        }
        auto it = by_vars.find(feats);
        int32_t r;
        if (it == by_vars.end()) {
            r = (int32_t)regions.size();
            regions.emplace_back();
            regions[r].leaf = true;
            regions[r].vars = feats;
            by_vars[feats] = r;
        } else {
            r = it->second;
        }
        region_of[u] = r;
        index_in[u] = (int32_t)regions[r].nodes.size();
        regions[r].nodes.push_back(u);
    }
    if (regions.empty()) return fail("no leaf regions");

    // ---- sum regions: sums with identical child sets
    std::unordered_map<uint64_t, std::vector<int32_t>> by_children;
    std::vector<int64_t> kids;
    std::vector<std::vector<int64_t>> region_kids;  // sorted child list per sum region
    std::vector<int32_t> sum_region_ids;
    for (int64_t u = 0; u < n; ++u) {
        if (c.kind[u] != SPN_SUM) continue;
        kids.assign(c.ch.begin() + c.cb[u], c.ch.begin() + c.cb[u + 1]);
        std::sort(kids.begin(), kids.end());
        if (std::adjacent_find(kids.begin(), kids.end()) != kids.end())
            return fail("sum with a repeated child");
        const uint64_t h = hash_vec(kids);
        int32_t r = -1;
        for (int32_t cand : by_children[h])
            if (region_kids[cand] == kids) r = cand;
        if (r < 0) {
            r = (int32_t)region_kids.size();
            region_kids.push_back(kids);
            by_children[h].push_back(r);
            sum_region_ids.push_back((int32_t)regions.size());
            regions.emplace_back();
        }
        const int32_t rid = sum_region_ids[r];
        region_of[u] = rid;
        index_in[u] = (int32_t)regions[rid].nodes.size();
        regions[rid].nodes.push_back(u);
    }

    // ---- partitions: products of two region values
    std::map<std::pair<int32_t, int32_t>, int32_t> by_pair;
    std::vector<Partition> parts;
    std::vector<int32_t> part_of(n, -1);
    std::vector<int32_t> cell_of(n, -1);
    for (int64_t u = 0; u < n; ++u) {
        if (c.kind[u] != SPN_PRODUCT || region_of[u] >= 0) continue;
        if (fan(u) != 2) return fail("inner product without two region children");
        int64_t a = c.ch[c.cb[u]], b = c.ch[c.cb[u] + 1];
        if (region_of[a] < 0 || region_of[b] < 0) return fail("product child outside regions");
        if (region_of[a] > region_of[b]) std::swap(a, b);
        if (region_of[a] == region_of[b]) return fail("product of one region with itself");
        const auto key = std::make_pair(region_of[a], region_of[b]);
        auto it = by_pair.find(key);
        int32_t p;
        if (it == by_pair.end()) {
            p = (int32_t)parts.size();
            parts.emplace_back();
            parts[p].ra = key.first;
            parts[p].rb = key.second;
            by_pair[key] = p;
        } else {
            p = it->second;
        }
        Partition &P = parts[p];
        const int64_t na = (int64_t)regions[P.ra].nodes.size(), nb = (int64_t)regions[P.rb].nodes.size();
        if (P.prods.empty()) P.prods.assign(na * nb, -1);
        const int64_t cell = (int64_t)index_in[a] * nb + index_in[b];
        if (P.prods[cell] >= 0) return fail("duplicate product in a partition");
        P.prods[cell] = u;
        part_of[u] = p;
        cell_of[u] = (int32_t)cell;
    }
    for (auto &P : parts)
        for (int64_t x : P.prods)
            if (x < 0) return fail("partition is not a complete cross product");
    // every region consumed by exactly one partition (except the root region)
    for (int32_t p = 0; p < (int32_t)parts.size(); ++p) {
        for (int32_t r : {parts[p].ra, parts[p].rb}) {
            if (regions[r].consumer_partition >= 0 && regions[r].consumer_partition != p)
                return fail("region consumed by two partitions");
            regions[r].consumer_partition = p;
        }
    }
    // region values consumed only by their partition's products
    for (int32_t r = 0; r < (int32_t)regions.size(); ++r)
        for (int64_t u : regions[r].nodes)
            for (int64_t e = c.pb[u]; e < c.pb[u + 1]; ++e)
                if (part_of[c.par[e]] != regions[r].consumer_partition)
                    return fail("region value with a foreign consumer");
    // sum regions: children = union of complete partitions
    for (size_t k = 0; k < region_kids.size(); ++k) {
        const int32_t rid = sum_region_ids[k];
        std::vector<int32_t> ps;
        for (int64_t ch : region_kids[k]) {
            if (part_of[ch] < 0) return fail("sum child is not a partition product");
            ps.push_back(part_of[ch]);
        }
        std::sort(ps.begin(), ps.end());
        ps.erase(std::unique(ps.begin(), ps.end()), ps.end());
        size_t total = 0;
        for (int32_t p : ps) {
            total += parts[p].prods.size();
            if (parts[p].consumer_region >= 0) return fail("partition consumed by two regions");
            parts[p].consumer_region = rid;
        }
        if (total != region_kids[k].size()) return fail("sum region covers a partial partition");
        regions[rid].partitions = ps;
    }
    // the roots: exactly the sums of one region, each root once
    const int32_t R0 = (int32_t)g.roots.size();
    int32_t root_region = -1;
    std::vector<int32_t> root_value(R0, -1);
    for (int64_t u = 0; u < n; ++u) {
        if (c.rootrefs[u].empty()) continue;
        if (c.kind[u] != SPN_SUM || region_of[u] < 0) return fail("root is not a layered sum");
        if (c.rootrefs[u].size() != 1) return fail("repeated root");
        if (root_region >= 0 && region_of[u] != root_region) return fail("roots in several regions");
        root_region = region_of[u];
    }
    if (root_region < 0) return fail("no root region");
    if ((int32_t)regions[root_region].nodes.size() != R0) return fail("root region has non-root sums");
    if (regions[root_region].consumer_partition >= 0) return fail("root region is consumed");
    for (int32_t r = 0; r < (int32_t)regions.size(); ++r)
        if (r != root_region && regions[r].consumer_partition < 0)
            return fail("dangling region");
    for (int32_t r = 0; r < (int32_t)regions.size(); ++r)
        if (!regions[r].leaf && r != root_region && regions[r].partitions.size() != 1)
            return fail("internal sum region with several partitions");
    for (auto &reg : regions) {
        if (reg.nodes.size() > 64) return fail("region with more than 64 values");
        if (reg.leaf && (reg.nodes.size() % 8 || reg.nodes.size() > 64))
            return fail("leaf region size must be a multiple of 8 (<= 64)");
        if (!reg.leaf && reg.nodes.size() < 1) return fail("empty region");
    }
    for (auto &P : parts) {
        const size_t na = regions[P.ra].nodes.size(), nb = regions[P.rb].nodes.size();
        if (na % 4 || nb > 64 || na > 60) return fail("region sizes need na % 4 == 0, <= 60");
        (void)nb;
    }

    // ---- build the schedule (post-order over each repetition's region tree)
    plan.F = g.F;
    plan.C = R0;
    plan.R = (int32_t)regions[root_region].partitions.size();
    std::vector<int32_t> root_order(R0);  // root region value index -> root index
    for (int64_t u : regions[root_region].nodes) root_order[index_in[u]] = c.rootrefs[u][0];
    const int TILE = 128;
    int32_t buf_top = 0, buf_peak = 0;
    std::vector<double> cvals;
    auto add_weights = [&](LStep &st, int32_t rid, int32_t p, bool root) {
        const Partition &P = parts[p];
        const int32_t na = (int32_t)regions[P.ra].nodes.size();
        const int32_t nb = (int32_t)regions[P.rb].nodes.size();
        const int32_t S = (int32_t)regions[rid].nodes.size();
        st.na = na;
        st.nb = nb;
        st.n_out = S;
        st.k_pad = (nb + 15) / 16 * 16;
        st.s_per_group = std::max(1, std::min(S, n_cap / na));
        // an even number of sums per group balances the two epilogue warp halves
        if (st.s_per_group > 1 && st.s_per_group < S && (st.s_per_group & 1)) st.s_per_group -= 1;
        st.n_groups = (S + st.s_per_group - 1) / st.s_per_group;
        st.n_group = (st.s_per_group * na + 15) / 16 * 16;
        st.w_group_bytes = (int64_t)st.n_group * st.k_pad * 2;
        // align the weight images to 16 bytes
        while (plan.wimg.size() % 8) plan.wimg.push_back(0);
        st.w_off = (int64_t)plan.wimg.size() * 2;
        // weights W[s][i][j] for value s of region rid (root: value index of the root)
        std::vector<double> W((size_t)S * na * nb, 0.0);
        for (int64_t sn : regions[rid].nodes) {
            const int32_t s = index_in[sn];
            for (int64_t e = c.cb[sn]; e < c.cb[sn + 1]; ++e) {
                const int64_t ch = c.ch[e];
                if (part_of[ch] != p) continue;
                const int32_t cell = cell_of[ch];
                W[(size_t)s * na * nb + cell] = c.w[e];  // cell = i * nb + j
            }
        }
        (void)root;
        for (double w : W) {
            plan.w_max = std::max(plan.w_max, w);
            if (w > 0.0 && (plan.w_min_nz == 0.0 || w < plan.w_min_nz)) plan.w_min_nz = w;
        }
        plan.raw.push_back(W);
        for (int32_t gi = 0; gi < st.n_groups; ++gi) {
            std::vector<uint16_t> hi((size_t)st.n_group * st.k_pad, 0), lo(hi.size(), 0);
            for (int32_t sl = 0; sl < st.s_per_group; ++sl) {
                const int32_t s = gi * st.s_per_group + sl;
                if (s >= S) break;
                for (int32_t i = 0; i < na; ++i)
                    for (int32_t j = 0; j < nb; ++j) {
                        const int32_t row = sl * na + i;  // N index
                        const double w = W[(size_t)s * na * nb + (size_t)i * nb + j];
                        const uint16_t h = f32_to_f16((float)w);
                        const uint16_t l = f32_to_f16((float)(w - (double)f16_to_f32(h)));
                        // K-major no-swizzle core-matrix image: (k/8)*LBO + (row/8)*128 + (row%8)*16 + (k%8)*2
                        const size_t lbo = (size_t)(st.n_group / 8) * 64;  // in f16 elements
                        const size_t idx = (size_t)(j / 8) * lbo + (size_t)(row / 8) * 64 +
                                           (size_t)(row % 8) * 8 + (size_t)(j % 8);
                        hi[idx] = h;
                        lo[idx] = l;
                    }
            }
            plan.wimg.insert(plan.wimg.end(), hi.begin(), hi.end());
            plan.wimg.insert(plan.wimg.end(), lo.begin(), lo.end());
        }
        plan.tc_flops_per_sample += 2LL * na * nb * S;
        plan.fma_per_sample += (int64_t)S * na;
        plan.mufu_per_sample += na + nb + S;
    };
    // Stack allocation of the activation buffers: a region's output is placed
    // at the stack top it was started with.  A SUM step reads its inputs only
    // in its first phase, so its output may overwrite them.
    std::function<int32_t(int32_t)> visit = [&](int32_t rid) -> int32_t {
        Region &reg = regions[rid];
        const int32_t top0 = buf_top;
        LStep st;
        memset(&st, 0, sizeof(st));
        if (reg.leaf) {
            st.type = 0;
            const int32_t I = (int32_t)reg.nodes.size();
            const int32_t V = (int32_t)reg.vars.size();
            st.n_out = I;
            st.n_vars = V;
            st.vars_off = (int64_t)plan.vars.size();
            plan.vars.insert(plan.vars.end(), reg.vars.begin(), reg.vars.end());
            // staged parameter block (16-byte aligned, one bulk copy):
            //   ab[v][g][k] = (a, b) float2 (see below), then C[i] (padded to a multiple of 4)
            while (plan.fparams.size() % 4) plan.fparams.push_back(0.f);
            st.par_off = (int64_t)plan.fparams.size();
            // (a, b) pairs grouped by the kernel's 8 distribution groups of
            // DPT = I/8: ab[v][g][k] = pair of distribution g*DPT + k, DPT
            // padded to even so a thread loads two pairs per LDS.128
            const int32_t DPT = I / 8, DPTp = DPT + (DPT & 1);
            std::vector<float> ab((size_t)V * 8 * DPTp * 2, 0.f);
            std::vector<double> Cs(I, 0.0);
            std::vector<double> raw((size_t)2 * V * I + I, 0.0);  // a[v][i], b[v][i], C[i]
            for (int32_t i = 0; i < I; ++i) {
                const int64_t u = reg.nodes[i];
                std::vector<int64_t> leaves;
                if (c.kind[u] == SPN_GAUSSIAN) leaves.push_back(u);
                else leaves.assign(c.ch.begin() + c.cb[u], c.ch.begin() + c.cb[u + 1]);
                for (int64_t lf : leaves) {
                    const int64_t o = c.orig[lf];
                    const int32_t f = g.feature[o];
                    const int32_t v = (int32_t)(std::lower_bound(reg.vars.begin(), reg.vars.end(), f) -
                                                reg.vars.begin());
                    const double *pp = g.params.data() + g.param_begin[o];
                    const double a = 1.0 / (pp[1] * std::sqrt(2.0 * M_LN2));
                    Cs[i] += -std::log2(pp[1] * std::sqrt(2.0 * M_PI));
                    const size_t idx = (((size_t)v * 8 + (size_t)(i / DPT)) * DPTp + (size_t)(i % DPT)) * 2;
                    ab[idx] = (float)a;
                    ab[idx + 1] = (float)(a * pp[0]);
                    raw[(size_t)v * I + i] = a;
                    raw[(size_t)V * I + (size_t)v * I + i] = a * pp[0];
                }
            }
            for (int32_t i = 0; i < I; ++i) raw[(size_t)2 * V * I + i] = Cs[i];
            plan.raw.push_back(std::move(raw));
            plan.child_a.push_back(-1);
            plan.child_b.push_back(-1);
            plan.fparams.insert(plan.fparams.end(), ab.begin(), ab.end());
            st.cst_off = (int64_t)plan.fparams.size();
            for (int32_t i = 0; i < I; ++i) plan.fparams.push_back((float)Cs[i]);
            while (plan.fparams.size() % 4) plan.fparams.push_back(0.f);
            st.w_off = (int64_t)plan.fparams.size() - st.par_off;  // LEAF: block size (floats)
            st.buf_out = top0;
            buf_top = top0 + I * TILE;
            buf_peak = std::max(buf_peak, buf_top);
            plan.fma_per_sample += 2LL * I * V;
            plan.n_leaf_regions++;
            plan.steps.push_back(st);
            return st.buf_out;
        }
        const Partition &P = parts[reg.partitions[0]];
        st.buf_a = visit(P.ra);
        const int32_t ca = (int32_t)plan.steps.size() - 1;
        st.buf_b = visit(P.rb);
        const int32_t cb = (int32_t)plan.steps.size() - 1;
        st.type = 1;
        add_weights(st, rid, reg.partitions[0], false);
        plan.child_a.push_back(ca);
        plan.child_b.push_back(cb);
        st.buf_out = top0;
        buf_top = top0 + st.n_out * TILE;
        buf_peak = std::max(buf_peak, buf_top);
        plan.n_sum_regions++;
        plan.steps.push_back(st);
        return st.buf_out;
    };
    for (int32_t p : regions[root_region].partitions) {
        const Partition &P = parts[p];
        const int32_t top0 = buf_top;
        LStep st;
        memset(&st, 0, sizeof(st));
        st.buf_a = visit(P.ra);
        const int32_t ca = (int32_t)plan.steps.size() - 1;
        st.buf_b = visit(P.rb);
        const int32_t cb = (int32_t)plan.steps.size() - 1;
        st.type = 2;
        add_weights(st, root_region, p, true);
        plan.child_a.push_back(ca);
        plan.child_b.push_back(cb);
        st.buf_out = -1;
        plan.steps.push_back(st);
        buf_top = top0;
    }
    // root values must be emitted in root-index order: remap via root_order
    plan.root_map = root_order;
    plan.smem_floats = buf_peak;
    int32_t next = -1;
    for (int32_t i = (int32_t)plan.steps.size() - 1; i >= 0; --i) {
        LStep &st = plan.steps[i];
        if (st.type == 0) {
            st.rep = next;
            next = i;
        }
    }
    plan.first_leaf = next;
    for (auto &st : plan.steps) {
        if (st.type == 0) {
            plan.max_vars = std::max(plan.max_vars, st.n_vars);
            plan.max_leaf_params = std::max<int32_t>(plan.max_leaf_params, (int32_t)st.w_off);
        }
        plan.max_kpad = std::max(plan.max_kpad, st.k_pad);
        plan.max_ngroup = std::max(plan.max_ngroup, st.n_group);
        plan.max_na = std::max(plan.max_na, st.na);
    }
    plan.ok = true;
}

// ---------------------------------------------------------------- v2 plan
void build_rat2(const LayeredPlan &lp, Rat2Plan &p, bool leaf_tc) {
    p = Rat2Plan();
    auto fail = [&](const std::string &why) {
        p.ok = false;
        p.why = why;
    };
    if (!lp.ok) return fail("not layered: " + lp.why);
    const int32_t ns = (int32_t)lp.steps.size();
    if ((int32_t)lp.child_a.size() != ns || (int32_t)lp.raw.size() != ns)
        return fail("layered plan without the region tree");
    // ---- step kinds, uniform widths
    std::vector<int32_t> kind(ns, 0);  // 0 LEAF, 1 BOT, 2 UP
    int32_t I = -1, S = -1;
    for (int32_t t = 0; t < ns; ++t) {
        const LStep &st = lp.steps[t];
        if (st.type == 0) {
            if (I >= 0 && st.n_out != I) return fail("leaf regions of different widths");
            I = st.n_out;
            continue;
        }
        const int32_t a = lp.child_a[t], b = lp.child_b[t];
        const bool la = lp.steps[a].type == 0, lb = lp.steps[b].type == 0;
        if (la != lb) return fail("partition of a leaf region and a sum region");
        kind[t] = la ? 1 : 2;
        if (st.type == 1) {
            if (S >= 0 && st.n_out != S) return fail("sum regions of different widths");
            S = st.n_out;
        }
    }
    if (I < 8 || I % 8 || I > 48) return fail("leaf width must be a multiple of 8, <= 48");
    if (S < 0) S = 0;
    if (S > 48) return fail("sum regions wider than 48");
    // ---- TMEM activation slots: a sum region at depth d (root region = 0)
    // writes slot d + (right child ? 1 : 0); its parent reads both children
    std::vector<int32_t> slot(ns, 0), depth(ns, 0);
    int32_t D = 0;
    for (int32_t t = ns - 1; t >= 0; --t) {  // parents come after children (post-order)
        const LStep &st = lp.steps[t];
        if (st.type == 0) continue;
        if (st.type == 2) depth[t] = 0;
        const int32_t a = lp.child_a[t], b = lp.child_b[t];
        depth[a] = depth[b] = depth[t] + 1;
        slot[a] = depth[t] + 1;
        slot[b] = depth[t] + 2;
        if (kind[t] == 2) D = std::max(D, depth[t] + 2);
    }
    p.F = lp.F;
    p.C = lp.C;
    p.I = I;
    p.S = S;
    p.D = D;
    // TMEM: two accumulators of R2_COLS_A + R2_COLS_B columns (tcgen05.mma
    // costs ~170 cycles per dependent step almost independently of N, so the
    // widest groups minimise the MMA count; the two chains interleave), then
    // the D activation slots and the C root accumulators
    const int32_t fixed_cols = D * S + p.C;
    const int32_t na_max = std::max(I, S);
    const int32_t CA = leaf_tc ? R2T_COLS_A : R2_COLS_A, CB = leaf_tc ? R2T_COLS_B : R2_COLS_B;
    const int32_t CL = leaf_tc ? R2T_COLS_L : 0;
    if (CA + CB + CL + fixed_cols > 512)
        return fail("TMEM budget: " + std::to_string(fixed_cols) + " activation/root columns");
    if (na_max > CB) return fail("region wider than an accumulator buffer");
    p.gcols = CA + CB + CL;
    p.cols_a = CA;
    p.cols_b = CB;
    p.leaf_tc = leaf_tc;
    if (leaf_tc) {
        int32_t vmax = 0;
        for (const LStep &st : lp.steps)
            if (st.type == 0) vmax = std::max(vmax, st.n_vars);
        p.lvp = (vmax + 3) / 4 * 4;
        p.kl_j = (2 * p.lvp + 1 + 15) / 16 * 16;
        p.kl_m = (3 * p.lvp + 15) / 16 * 16;
    }
    p.ea_max = (na_max + 7) / 8 * 8;
    p.kpad_bot = (I + 15) / 16 * 16;
    p.kpad_up = S > 0 ? (S + 15) / 16 * 16 : 16;
    // ---- steps (and the single-pass error bound, log2 units, per step)
    std::vector<double> err(ns, 0.0);
    double err_root = 0.0;
    for (int32_t t = 0; t < ns; ++t) {
        const LStep &st = lp.steps[t];
        R2Step r;
        memset(&r, 0, sizeof(r));
        r.type = kind[t];
        r.n_out = st.n_out;
        r.slot_out = st.type == 1 ? slot[t] : 0;
        r.root = st.type == 2 ? 1 : 0;
        if (st.type == 0 && leaf_tc) {
            // tensor-core leaf layer: centres M_v, the joint and marginal
            // parameter images (B operand, K-major, N = R2T_COLS_L rows)
            const int32_t V = st.n_vars, NL = R2T_COLS_L, lvp = p.lvp;
            r.n_vars = V;
            r.vars_off = (int64_t)p.vars.size();
            p.vars.insert(p.vars.end(), lp.vars.begin() + st.vars_off,
                          lp.vars.begin() + st.vars_off + V);
            const std::vector<double> &raw = lp.raw[t];
            while (p.fparams.size() % 4) p.fparams.push_back(0.f);
            r.blk_off = (int64_t)p.fparams.size();
            std::vector<float> M(lvp, 0.f);
            for (int32_t v = 0; v < V; ++v) {  // midpoint of the region's means on variable v
                double lo = INFINITY, hi = -INFINITY;
                for (int32_t i = 0; i < I; ++i) {
                    const double mu = raw[(size_t)V * I + (size_t)v * I + i] / raw[(size_t)v * I + i];
                    lo = std::min(lo, mu);
                    hi = std::max(hi, mu);
                }
                M[v] = (float)(0.5 * (lo + hi));
                if (!std::isfinite(M[v])) return fail("leaf tensor cores: non-finite centre");
            }
            p.fparams.insert(p.fparams.end(), M.begin(), M.end());
            r.blk_floats = lvp;
            // P[k][i]: k = 2v -a^2, 2v+1 2 a b~, then the constant column
            // sum_v (c_v - b~^2) (joint) or per-variable c_v - b~^2 (marginal)
            const double K0 = 0.5 * std::log2(M_LN2 / M_PI);  // c_v = log2(a) + K0
            std::vector<double> Pj((size_t)p.kl_j * NL, 0.0), Pm((size_t)p.kl_m * NL, 0.0);
            for (int32_t i = 0; i < I; ++i) {
                double cj = 0.0;
                for (int32_t v = 0; v < V; ++v) {
                    const double a = raw[(size_t)v * I + i], b = raw[(size_t)V * I + (size_t)v * I + i];
                    const double bt = b - a * (double)M[v];
                    const double pq = -a * a, px = 2.0 * a * bt, pz = std::log2(a) + K0 - bt * bt;
                    Pj[(size_t)(2 * v) * NL + i] = Pm[(size_t)(2 * v) * NL + i] = pq;
                    Pj[(size_t)(2 * v + 1) * NL + i] = Pm[(size_t)(2 * v + 1) * NL + i] = px;
                    Pm[(size_t)(2 * lvp + v) * NL + i] = pz;
                    cj += pz;
                }
                Pj[(size_t)(2 * lvp) * NL + i] = cj;
            }
            while (p.wimg.size() % 64) p.wimg.push_back(0);  // 128-byte aligned images
            r.w_off = (int64_t)p.wimg.size() * 2;
            r.wbytes_a = (int64_t)NL * p.kl_j * 2;
            r.wbytes_b = (int64_t)NL * p.kl_m * 2;
            for (int pass = 0; pass < 2; ++pass) {
                const std::vector<double> &P = pass ? Pm : Pj;
                const int32_t K = pass ? p.kl_m : p.kl_j;
                std::vector<uint16_t> hi((size_t)NL * K, 0), lo((size_t)NL * K, 0);
                for (int32_t k = 0; k < K; ++k)
                    for (int32_t n = 0; n < NL; ++n) {
                        const double v = P[(size_t)k * NL + n];
                        if (!(std::fabs(v) < 60000.0)) return fail("leaf tensor cores: constant outside f16");
                        const uint16_t h = f32_to_f16((float)v);
                        const size_t idx = (size_t)(k / 8) * ((size_t)NL / 8) * 64 + (size_t)(n / 8) * 64 +
                                           (size_t)(n % 8) * 8 + (size_t)(k % 8);
                        hi[idx] = h;
                        lo[idx] = f32_to_f16((float)(v - (double)f16_to_f32(h)));
                    }
                p.wimg.insert(p.wimg.end(), hi.begin(), hi.end());
                p.wimg.insert(p.wimg.end(), lo.begin(), lo.end());
            }
            p.max_vars = std::max(p.max_vars, V);
            p.max_blk = std::max<int32_t>(p.max_blk, (int32_t)r.blk_floats);
            p.n_leaf++;
            p.steps.push_back(r);
            continue;
        }
        if (st.type == 0) {
            const int32_t V = st.n_vars;
            r.n_vars = V;
            r.vars_off = (int64_t)p.vars.size();
            p.vars.insert(p.vars.end(), lp.vars.begin() + st.vars_off,
                          lp.vars.begin() + st.vars_off + V);
            // block: (a, b)[v][i] interleaved, then C[i]; 16-byte multiple
            while (p.fparams.size() % 4) p.fparams.push_back(0.f);
            r.blk_off = (int64_t)p.fparams.size();
            const std::vector<double> &raw = lp.raw[t];
            for (int32_t v = 0; v < V; ++v)
                for (int32_t i = 0; i < I; ++i) {
                    p.fparams.push_back((float)raw[(size_t)v * I + i]);
                    p.fparams.push_back((float)raw[(size_t)V * I + (size_t)v * I + i]);
                }
            for (int32_t i = 0; i < I; ++i) p.fparams.push_back((float)raw[(size_t)2 * V * I + i]);
            while (p.fparams.size() % 4) p.fparams.push_back(0.f);
            r.blk_floats = (int64_t)p.fparams.size() - r.blk_off;
            p.max_vars = std::max(p.max_vars, V);
            p.max_blk = std::max<int32_t>(p.max_blk, (int32_t)r.blk_floats);
            p.n_leaf++;
            p.steps.push_back(r);
            continue;
        }
        const int32_t na = st.na, nb = st.nb, n_out = st.n_out;
        r.na = na;
        r.nb = nb;
        r.kpad = (nb + 15) / 16 * 16;
        if (r.type == 2) {
            r.slot_a = slot[lp.child_a[t]];
            r.slot_b = slot[lp.child_b[t]];
        }
        // sums per group: the most whose columns (x16) fit the buffer
        auto cap = [&](int32_t cols) {
            int32_t c = cols / na;
            while (c > 1 && (c * na + 15) / 16 * 16 > cols) --c;
            return std::max(1, c);
        };
        const int32_t cap_a = cap(CA), cap_b = cap(CB);
        int32_t spg_a = cap_a, spg_b = cap_b;
        if (n_out <= cap_a + cap_b) {  // one pair: split in proportion to the buffers
            spg_a = std::min(cap_a, (n_out * cap_a + cap_a + cap_b - 1) / (cap_a + cap_b));
            spg_b = n_out - spg_a;
            if (spg_b > cap_b) {
                spg_b = cap_b;
                spg_a = n_out - cap_b;
            }
        }
        const int32_t n_pairs = (n_out + spg_a + spg_b - 1) / (spg_a + spg_b);
        r.n_groups = 2 * n_pairs;
        r.spg_a = spg_a;
        r.spg_b = spg_b;
        r.ncol_a = std::max(16, (spg_a * na + 15) / 16 * 16);
        r.ncol_b = std::max(16, (spg_b * na + 15) / 16 * 16);
        // per-sum scale exponents: w' = w 2^k with max_ij w' in [1, 2)
        const std::vector<double> &W = lp.raw[t];
        while (p.fparams.size() % 4) p.fparams.push_back(0.f);
        r.blk_off = (int64_t)p.fparams.size();
        std::vector<double> scale(n_out, 1.0);
        double eps_step = 0.0;  // largest relative error of one of this step's sums
        for (int32_t s2 = 0; s2 < n_out; ++s2) {
            double mx = 0.0, mn = INFINITY, tot = 0.0;
            for (int64_t c = 0; c < (int64_t)na * nb; ++c) {
                const double w = W[(size_t)s2 * na * nb + c];
                mx = std::max(mx, w);
                mn = std::min(mn, w);
                tot += w;
            }
            const int k = mx > 0.0 ? -(int)std::floor(std::log2(mx)) : 0;
            scale[s2] = std::ldexp(1.0, k);
            p.fparams.push_back((float)k);
            double ew = 0.0;  // exact relative rounding of the f16 weights of this sum
            for (int64_t c = 0; c < (int64_t)na * nb; ++c) {
                const double w = W[(size_t)s2 * na * nb + c] * scale[s2];
                if (w > 0.0) ew = std::max(ew, std::fabs((double)f16_to_f32(f32_to_f16((float)w)) - w) / w);
            }
            const double rho = mn > 0.0 ? tot / mn : INFINITY;
            const double u16 = std::ldexp(1.0, -11), u32 = std::ldexp(1.0, -24);
            const double delta = (1.0 + ew) * (1.0 + u16) - 1.0 + std::ldexp(rho, -29) +
                                 (double)(nb + na + 8) * u32;
            eps_step = std::max(eps_step, delta < 0.5 ? -std::log1p(-delta) / M_LN2 : INFINITY);
        }
        err[t] = eps_step + err[lp.child_a[t]] + err[lp.child_b[t]];
        if (st.type == 2) err_root = std::max(err_root, err[t]);
        while (p.fparams.size() % 4) p.fparams.push_back(0.f);
        r.wbytes_a = (int64_t)r.ncol_a * r.kpad * 2;
        r.wbytes_b = (int64_t)r.ncol_b * r.kpad * 2;
        while (p.wimg.size() % 64) p.wimg.push_back(0);  // 128-byte aligned images
        r.w_off = (int64_t)p.wimg.size() * 2;
        for (int32_t gi = 0; gi < r.n_groups; ++gi) {
            const bool gb = gi & 1;
            const int32_t ncol = gb ? r.ncol_b : r.ncol_a, spg = gb ? spg_b : spg_a;
            const int32_t s_first = (gi / 2) * (spg_a + spg_b) + (gb ? spg_a : 0);
            const size_t gel = (size_t)ncol * r.kpad;
            std::vector<uint16_t> hi(gel, 0), lo(gel, 0);
            for (int32_t sl = 0; sl < spg; ++sl) {
                const int32_t s2 = s_first + sl;
                if (s2 >= n_out) break;
                for (int32_t i = 0; i < na; ++i)
                    for (int32_t j = 0; j < nb; ++j) {
                        const int32_t row = sl * na + i;
                        const double w = W[(size_t)s2 * na * nb + (size_t)i * nb + j] * scale[s2];
                        const uint16_t h = f32_to_f16((float)w);
                        const uint16_t l = f32_to_f16((float)(w - (double)f16_to_f32(h)));
                        const size_t idx = (size_t)(j / 8) * ((size_t)ncol / 8) * 64 +
                                           (size_t)(row / 8) * 64 + (size_t)(row % 8) * 8 +
                                           (size_t)(j % 8);
                        hi[idx] = h;
                        lo[idx] = l;
                    }
            }
            p.wimg.insert(p.wimg.end(), hi.begin(), hi.end());
            p.wimg.insert(p.wimg.end(), lo.begin(), lo.end());
        }
        p.max_wgroup = std::max<int32_t>(p.max_wgroup, (int32_t)std::max(r.wbytes_a, r.wbytes_b));
        p.n_sum++;
        p.steps.push_back(r);
    }
    p.root_map = lp.root_map;
    p.tc_err_1pass = err_root * M_LN2;
    p.ok = true;
}

}  // namespace spnb
