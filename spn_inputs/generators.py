"""Seeded synthetic SPN generators shaped like the paper's workloads.

No inference arithmetic lives here: only structure, parameters and
(in ``sampling.py``) ancestral sampling of data.  Recipes follow SURVEY.md
Appendix A/B and §8(d); DESIGN.md §"Input recipe" restates them.

* ``toy_spn``        -- config 1, the 3-variable discrete SPN standing in for
                        the absent Fig. 1.
* ``speaker_spn``    -- config 2/3, LearnSPN-like Gaussian tree over 26
                        MFCC-like features (~2569 ops, ~49%
                        Gaussian leaves).
* ``rat_spn``        -- config 4/5, RAT-SPN region graph (PAPER.md L461-479:
                        ~165k leaves / ~170k products / >3k sums per class).
* ``tiny_discrete_spn`` -- B3, small normalised discrete SPNs for brute force.
"""
from __future__ import annotations

import numpy as np

from .graph import (FlatSPN, GraphBuilder, disjoint_union, SUM, PRODUCT,
                    GAUSSIAN)


# --------------------------------------------------------------------------
# Config 1: toy SPN
# --------------------------------------------------------------------------
def toy_spn() -> FlatSPN:
    """S0 = 0.3 P0 + 0.7 P1
    P0 = Cat_a(X0;[.2,.8]) * S1 * Hist_d(X2;[(0,2,.1),(2,4,.4)])
    S1 = 0.4 Cat_b(X1;[.5,.3,.2]) + 0.6 Cat_c(X1;[.1,.2,.7])
    P1 = Cat_e(X0;[.6,.4]) * P2
    P2 = Cat_f(X1;[.3,.3,.4]) * Hist_g(X2;[(0,1,.25),(1,3,.125),(3,4,.5)])
    2 sums, 3 products, 5 categorical + 2 histogram leaves (12 nodes)."""
    b = GraphBuilder(3)
    cat_a = b.categorical(0, [0.2, 0.8])
    cat_b = b.categorical(1, [0.5, 0.3, 0.2])
    cat_c = b.categorical(1, [0.1, 0.2, 0.7])
    hist_d = b.histogram(2, [(0, 2, 0.1), (2, 4, 0.4)])
    cat_e = b.categorical(0, [0.6, 0.4])
    cat_f = b.categorical(1, [0.3, 0.3, 0.4])
    hist_g = b.histogram(2, [(0, 1, 0.25), (1, 3, 0.125), (3, 4, 0.5)])
    s1 = b.sum([cat_b, cat_c], [0.4, 0.6])
    p0 = b.product([cat_a, s1, hist_d])
    p2 = b.product([cat_f, hist_g])
    p1 = b.product([cat_e, p2])
    s0 = b.sum([p0, p1], [0.3, 0.7])
    return b.build([s0], meta={"name": "toy", "domains": [2, 3, 4]})


# --------------------------------------------------------------------------
# Config 2/3: speaker-ID-shaped SPN
# --------------------------------------------------------------------------
def _speaker_once(rng, F, sum_k, prod_k):
    b = GraphBuilder(F)

    def build(scope, is_sum):
        if len(scope) == 1:
            f = int(scope[0])
            return b.gaussian(f, float(rng.normal(0.0, 1.0)),
                              float(rng.uniform(0.2, 2.0)))
        if is_sum:
            k = int(rng.integers(sum_k[0], sum_k[1] + 1))
            ch = [build(scope, False) for _ in range(k)]
            w = rng.dirichlet(np.ones(k))
            return b.sum(ch, w)
        perm = rng.permutation(scope)
        g = int(rng.integers(prod_k[0], prod_k[1] + 1))
        g = min(g, len(perm))
        cuts = np.sort(rng.choice(np.arange(1, len(perm)), size=g - 1, replace=False))
        groups = np.split(perm, cuts)
        ch = [build(grp, True) for grp in groups]
        return b.product(ch)

    root = build(np.arange(F), True)
    return b.build([root])


def speaker_spn(seed: int, F: int = 26, sum_k=(2, 3), prod_k=(2, 4),
                lo: int = 1800, hi: int = 3000) -> FlatSPN:
    """LearnSPN-like tree.  Root is a sum; sums have 2-3 product children
    over the same scope; products split a random permutation of their scope
    into 2-4 contiguous groups; a size-1 group is a Gaussian leaf, otherwise
    a sum.  mu ~ N(0,1), sigma ~ U[0.2, 2], weights ~ Dirichlet(1).  Redraws
    until the node count is in [lo, hi] (paper average 2569 ops, L394)."""
    rng = np.random.default_rng(seed)
    for attempt in range(1000):
        g = _speaker_once(rng, F, sum_k, prod_k)
        if lo <= g.n_nodes <= hi:
            g.meta.update({"name": "speaker", "seed": seed, "attempt": attempt})
            return g
    raise RuntimeError("speaker_spn: no graph in node range")


def speaker_set(seeds, F: int = 26) -> FlatSPN:
    """Config 3: one SPN per speaker, as a multi-root union."""
    g = disjoint_union([speaker_spn(s, F) for s in seeds])
    g.meta.update({"name": "speaker_set", "seeds": list(seeds)})
    return g


# --------------------------------------------------------------------------
# B3: tiny normalised discrete SPNs (brute-force pins)
# --------------------------------------------------------------------------
def tiny_discrete_spn(seed: int, n_vars: int = 3, max_states: int = 4,
                      use_histograms: bool = True) -> FlatSPN:
    """Small complete + decomposable SPN with categorical / histogram leaves
    (normalised weights and leaves), so the sum over all assignments is 1."""
    rng = np.random.default_rng(seed)
    domains = [int(rng.integers(2, max_states + 1)) for _ in range(n_vars)]
    b = GraphBuilder(n_vars)

    def leaf(f):
        K = domains[f]
        if use_histograms and rng.random() < 0.4 and K >= 2:
            # random integer bucket boundaries covering [0, K)
            n_b = int(rng.integers(1, K + 1))
            inner = np.sort(rng.choice(np.arange(1, K), size=n_b - 1, replace=False)) if n_b > 1 else np.array([], dtype=int)
            edges = [0] + [int(e) for e in inner] + [K]
            mass = rng.dirichlet(np.ones(n_b))
            bk = [(edges[i], edges[i + 1], float(mass[i] / (edges[i + 1] - edges[i])))
                  for i in range(n_b)]
            return b.histogram(f, bk)
        return b.categorical(f, rng.dirichlet(np.ones(K)))

    def build(scope, is_sum, depth):
        if len(scope) == 1 and (not is_sum or depth > 2 or rng.random() < 0.5):
            return leaf(int(scope[0]))
        if is_sum:
            k = int(rng.integers(2, 4))
            ch = [build(scope, False, depth + 1) for _ in range(k)]
            return b.sum(ch, rng.dirichlet(np.ones(k)))
        if len(scope) == 1:
            return leaf(int(scope[0]))
        perm = rng.permutation(scope)
        g = int(rng.integers(2, len(perm) + 1))
        cuts = np.sort(rng.choice(np.arange(1, len(perm)), size=g - 1, replace=False))
        return b.product([build(grp, True, depth + 1) for grp in np.split(perm, cuts)])

    root = build(np.arange(n_vars), True, 0)
    return b.build([root], meta={"name": "tiny_discrete", "domains": domains,
                                 "seed": seed})


def tiny_gaussian_spn(seed: int, n_vars: int = 2) -> FlatSPN:
    """Small Gaussian SPN (for quadrature pins of marginals)."""
    rng = np.random.default_rng(seed)
    b = GraphBuilder(n_vars)

    def build(scope, is_sum, depth):
        if len(scope) == 1 and (not is_sum or depth > 1):
            f = int(scope[0])
            return b.gaussian(f, float(rng.normal()), float(rng.uniform(0.3, 1.5)))
        if is_sum:
            k = int(rng.integers(2, 4))
            return b.sum([build(scope, False, depth + 1) for _ in range(k)],
                         rng.dirichlet(np.ones(k)))
        if len(scope) == 1:
            f = int(scope[0])
            return b.gaussian(f, float(rng.normal()), float(rng.uniform(0.3, 1.5)))
        perm = rng.permutation(scope)
        return b.product([build(grp, True, depth + 1)
                          for grp in np.array_split(perm, 2)])

    root = build(np.arange(n_vars), True, 0)
    return b.build([root], meta={"name": "tiny_gaussian", "seed": seed})


# --------------------------------------------------------------------------
# Config 4/5: RAT-SPN
# --------------------------------------------------------------------------
def rat_spn(seed: int, F: int = 784, D: int = 5, R: int = 8, S: int = 20,
            I: int = 40, C: int = 10) -> FlatSPN:
    """RAT-SPN as a flat DAG (the shape SPFlow produces after conversion,
    PAPER.md L479).  Per repetition the F variables are split recursively
    into two random halves D times (2^D leaf regions).  A leaf region holds I
    factorised Gaussians (a product of one Gaussian leaf per variable).  A
    partition's products are the cross product of its two child regions'
    nodes (I^2 at the bottom, S^2 above).  Internal regions hold S sums over
    all products of their partition; the root region holds C sums over the
    R*S^2 top products of all repetitions.
    mu ~ U[0,1], sigma ~ U[0.1,1], weights = softmax(N(0,1)).

    Node ids are emitted bottom-up (children before parents) with numpy
    arrays, so C5-sized graphs (3.2M nodes, 31M edges) build in seconds.
    ``meta['rat']`` records the structure for the data sampler and for
    tests; the preparer never reads it (it detects layers from the DAG)."""
    rng = np.random.default_rng(seed)
    kinds = []      # list of (kind array chunk)
    feats = []
    nch = []
    params_chunks = []
    npar = []
    child_chunks = []
    weight_chunks = []
    n_nodes = 0

    def emit(kind, feature, n_children, children, weights, params, n_params):
        nonlocal n_nodes
        cnt = len(kind)
        kinds.append(kind)
        feats.append(feature)
        nch.append(n_children)
        child_chunks.append(children)
        weight_chunks.append(weights)
        params_chunks.append(params)
        npar.append(n_params)
        first = n_nodes
        n_nodes += cnt
        return np.arange(first, first + cnt, dtype=np.int64)

    def softmax_rows(shape):
        z = rng.normal(size=shape)
        z = np.exp(z - z.max(axis=-1, keepdims=True))
        return z / z.sum(axis=-1, keepdims=True)

    rep_info = []
    top_products = []   # per rep: ids [S*S] of the top partition's products
    for r in range(R):
        perm = rng.permutation(F)
        # region tree: list per depth of arrays of variable index sets
        regions = [[perm]]
        for d in range(D):
            nxt = []
            for reg in regions[-1]:
                h = len(reg) // 2
                sub = rng.permutation(reg)
                nxt.append(np.sort(sub[:h]))
                nxt.append(np.sort(sub[h:]))
            regions.append(nxt)
        # leaf regions at depth D: I factorised Gaussians each
        level_nodes = []   # per region at current depth: ids of its nodes
        leaf_info = []
        for reg in regions[D]:
            V = len(reg)
            mu = rng.uniform(0.0, 1.0, size=(I, V))
            sd = rng.uniform(0.1, 1.0, size=(I, V))
            lids = emit(np.full(I * V, GAUSSIAN, np.int32),
                        np.tile(reg.astype(np.int32), I),
                        np.zeros(I * V, np.int32),
                        np.zeros(0, np.int64), np.zeros(0, np.float64),
                        np.stack([mu.reshape(-1), sd.reshape(-1)], axis=1).reshape(-1),
                        np.full(I * V, 2, np.int32))
            pids = emit(np.full(I, PRODUCT, np.int32), np.full(I, -1, np.int32),
                        np.full(I, V, np.int32), lids.copy(),
                        np.zeros(I * V, np.float64), np.zeros(0, np.float64),
                        np.zeros(I, np.int32))
            level_nodes.append(pids)
            leaf_info.append({"vars": reg, "mu": mu, "sd": sd})
        sum_weights = []
        # internal levels D-1 .. 1 (sums), level 0 handled by the root
        for d in range(D - 1, -1, -1):
            new_level = []
            lvl_w = []
            for j in range(len(regions[d])):
                a = level_nodes[2 * j]
                bb = level_nodes[2 * j + 1]
                na, nb = len(a), len(bb)
                ch = np.stack([np.repeat(a, nb), np.tile(bb, na)], axis=1).reshape(-1)
                prods = emit(np.full(na * nb, PRODUCT, np.int32),
                             np.full(na * nb, -1, np.int32),
                             np.full(na * nb, 2, np.int32), ch,
                             np.zeros(2 * na * nb, np.float64),
                             np.zeros(0, np.float64), np.zeros(na * nb, np.int32))
                if d == 0:
                    top_products.append(prods)
                    new_level.append(prods)
                    continue
                w = softmax_rows((S, na * nb))
                sids = emit(np.full(S, SUM, np.int32), np.full(S, -1, np.int32),
                            np.full(S, na * nb, np.int32), np.tile(prods, S),
                            w.reshape(-1), np.zeros(0, np.float64),
                            np.zeros(S, np.int32))
                new_level.append(sids)
                lvl_w.append(w)
            level_nodes = new_level
            sum_weights.append(lvl_w)
        rep_info.append({"regions": regions, "leaves": leaf_info,
                         "sum_weights": sum_weights})
    # root region: C sums over the R*S^2 top products
    allp = np.concatenate(top_products)
    wr = softmax_rows((C, len(allp)))
    roots = emit(np.full(C, SUM, np.int32), np.full(C, -1, np.int32),
                 np.full(C, len(allp), np.int32), np.tile(allp, C),
                 wr.reshape(-1), np.zeros(0, np.float64), np.zeros(C, np.int32))

    kind = np.concatenate(kinds).astype(np.int32)
    n_children = np.concatenate(nch).astype(np.int32)
    n_params = np.concatenate(npar).astype(np.int32)
    child_begin = np.zeros(len(kind), np.int64)
    np.cumsum(n_children[:-1], out=child_begin[1:])
    param_begin = np.zeros(len(kind), np.int64)
    np.cumsum(n_params[:-1], out=param_begin[1:])
    g = FlatSPN(kind=kind, feature=np.concatenate(feats).astype(np.int32),
                child_begin=child_begin, n_children=n_children,
                param_begin=param_begin, n_params=n_params,
                children=np.concatenate(child_chunks).astype(np.int64),
                weights=np.concatenate(weight_chunks).astype(np.float64),
                params=np.concatenate(params_chunks).astype(np.float64),
                roots=roots, n_features=F,
                meta={"name": "rat", "seed": seed,
                      "rat": {"F": F, "D": D, "R": R, "S": S, "I": I, "C": C,
                              "reps": rep_info, "root_weights": wr}})
    return g


def rat_counts(F, D, R, S, I, C):
    """Closed-form node counts."""
    leaves = R * F * I
    n = [S] * D + [I]  # n[d] = nodes per region at depth d (d=D leaf regions)
    prods = R * (2 ** D) * I + sum(R * (2 ** d) * n[d + 1] ** 2 for d in range(D))
    sums = R * (2 ** D - 2) * S + C
    return {"leaves": leaves, "products": prods, "sums": sums,
            "nodes": leaves + prods + sums}


# --------------------------------------------------------------------------
# Named configs (BASELINE.json "configs")
# --------------------------------------------------------------------------
CONFIGS = {
    "C1": dict(desc="toy SPN (Fig.1 stand-in), 100k samples",
               n_samples=100_000),
    "C2": dict(desc="speaker-ID SPN, 26 Gaussian features, ~2.5k nodes, 1M samples",
               n_samples=1_000_000, graph_seed=2001, data_seed=2002),
    "C3": dict(desc="32 speaker SPNs, 20% NaN, argmax, 1M samples",
               n_samples=1_000_000, graph_seeds=list(range(3001, 3033)),
               data_seed=3002, nan_seed=3100, nan_p=0.2),
    "C4": dict(desc="RAT-SPN D5 R8 S20 I40 C10 over 784 features, 100k samples",
               n_samples=100_000, graph_seed=4001, data_seed=4002,
               rat=dict(F=784, D=5, R=8, S=20, I=40, C=10)),
    "C5": dict(desc="RAT-SPN D5 R50 S20 I40 C10 (3.24M nodes), 10M samples, argmax",
               n_samples=10_000_000, graph_seed=5001, data_seed=5002,
               rat=dict(F=784, D=5, R=50, S=20, I=40, C=10)),
}


def config_graph(name: str) -> FlatSPN:
    c = CONFIGS[name]
    if name == "C1":
        return toy_spn()
    if name == "C2":
        return speaker_spn(c["graph_seed"])
    if name == "C3":
        return speaker_set(c["graph_seeds"])
    return rat_spn(c["graph_seed"], **c["rat"])
