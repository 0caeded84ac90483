"""Compiled path (kernel KS): the code generator checked on CPU.

The generator builds an SSA IR per task and prints it as PTX (what the
library assembles for sm_100a) and as plain C++ with the same fp32
operations.  Here the C++ form is compiled with g++ and run against the fp64
oracle on the same seeded inputs (so the generator's arithmetic -- leaf
expansion, bias pushing of the sum weights, the LSE network, marginal
handling, task splitting, argmax -- is pinned without a GPU); the PTX form is
assembled with nvJitLink for sm_100a to check it is valid.  GPU parity of
the assembled kernels is in test_gpu_parity.py."""
import ctypes
import itertools
import os
import shutil
import subprocess
import tempfile

import numpy as np
import pytest

import paper_conf_cgo_sommera022_b200 as spnb
from oracle import oracle_eval
from spn_inputs import (toy_spn, toy_data, speaker_spn, speaker_set, rat_spn, tiny_discrete_spn,
                        tiny_gaussian_spn, ancestral_sample, add_outliers, nan_mask)

TOL = 1e-4
pytestmark = pytest.mark.skipif(shutil.which("g++") is None, reason="needs g++")


@pytest.fixture(scope="module", autouse=True)
def _lib():
    from paper_conf_cgo_sommera022_b200.build import build
    build()
    spnb.load_library()


_tmp = tempfile.mkdtemp(prefix="spnb_cg_")
_count = itertools.count()   # unique .so names: dlopen caches by path


def host_eval(g, x, marginal, space=0):
    """Run every generated task's C++ form over x; returns (out, argmax or None)."""
    G = spnb.Graph(g)
    first = spnb.codegen(G, 0, space=space)
    R = g.n_roots
    out = np.full((len(x), R), np.nan, np.float32)
    am = np.zeros(len(x), np.int32)
    xx = np.ascontiguousarray(x, np.float32)
    for t in range(first["n_tasks"]):
        cg = spnb.codegen(G, t, space=space)
        base = os.path.join(_tmp, f"t{os.getpid()}_{next(_count)}")
        with open(base + ".cpp", "w") as f:
            f.write(cg["source"])
        r = subprocess.run(["g++", "-O1", "-std=c++17", "-shared", "-fPIC", "-ffp-contract=off",
                            base + ".cpp", "-o", base + ".so"], capture_output=True, text=True)
        assert r.returncode == 0, r.stderr[:2000]
        fn = getattr(ctypes.CDLL(base + ".so"), cg["name"] + "_host")
        fn(xx.ctypes.data_as(ctypes.c_void_p), ctypes.c_longlong(len(x)),
           ctypes.c_longlong(x.shape[1]), out.ctypes.data_as(ctypes.c_void_p), ctypes.c_int(R),
           am.ctypes.data_as(ctypes.c_void_p) if first["n_tasks"] == 1 else None,
           cg["tables"].ctypes.data_as(ctypes.c_void_p), ctypes.c_int(int(marginal)))
    return out, (am if first["n_tasks"] == 1 else None), first["n_tasks"]


def _cmp(got, ref, tol=TOL):
    got = got.astype(np.float64)
    both_nan = np.isnan(got) & np.isnan(ref)
    both_inf = np.isneginf(got) & np.isneginf(ref)
    with np.errstate(invalid="ignore"):
        err = np.abs(got - ref) / np.maximum(1.0, np.abs(ref))
        ok = both_nan | both_inf | (err <= tol)
    assert ok.all(), f"{(~ok).sum()} mismatches: got {got[~ok][:3]} ref {ref[~ok][:3]}"


def _check(g, x, marginal=False, space=0):
    out, am, nt = host_eval(g, x, marginal, space)
    ref, am_ref = oracle_eval(g, x, marginal=marginal)
    _cmp(out, ref)
    if am is not None and g.n_roots > 1:
        s = np.sort(np.where(np.isnan(ref), -np.inf, ref), axis=1)
        decided = (s[:, -1] - s[:, -2]) > 2 * TOL * np.maximum(1.0, np.abs(s[:, -1]))
        assert np.array_equal(am[decided], am_ref[decided])
    return nt


def test_toy_joint_marginal():
    x = toy_data(3000, seed=3)
    _check(toy_spn(), x)
    _check(toy_spn(), nan_mask(x, 0.3, 4), marginal=True)


def test_speaker_joint_marginal_outliers_and_infinities():
    g = speaker_spn(2001)
    x, _ = ancestral_sample(g, 2000, 5)
    x = add_outliers(x, 0.02, 6)
    x[0, 3], x[1, 4], x[2, :] = np.inf, -np.inf, np.nan
    _check(g, x)
    _check(g, nan_mask(x, 0.2, 7), marginal=True)


def test_far_means_use_direct_form():
    """Leaves far from the per-feature centre (|b~| > 8) take the direct
    (a x - b)^2 form; accuracy must hold for means ~1e3 sigma apart."""
    from spn_inputs import GraphBuilder
    b = GraphBuilder(2)
    p0 = b.product([b.gaussian(0, -500.0, 0.5), b.gaussian(1, 3.0, 1.0)])
    p1 = b.product([b.gaussian(0, 700.0, 2.0), b.gaussian(1, -2.0, 0.25)])
    g = b.build([b.sum([p0, p1], [0.25, 0.75])])
    rng = np.random.default_rng(8)
    x = np.stack([np.where(rng.random(500) < 0.5, rng.normal(-500, 0.5, 500),
                           rng.normal(700, 2.0, 500)), rng.normal(0, 2, 500)], 1).astype(np.float32)
    _check(g, x)
    _check(g, nan_mask(x, 0.3, 9), marginal=True)


def test_multi_task_speaker_set():
    g = speaker_set([3001, 3002, 3003])
    x, _ = ancestral_sample(g, 1500, 10)
    assert _check(g, x) == 3   # three components, one task each (cap 3000 nodes)
    _check(g, nan_mask(x, 0.2, 11), marginal=True)


def test_single_task_argmax_fused():
    g = speaker_set([3001, 3002, 3003])
    G = spnb.Graph(g)
    assert spnb.codegen(G, 0)["n_tasks"] == 3
    g2 = speaker_set([3004])
    _check(g2, ancestral_sample(g2, 500, 12)[0])


def test_shared_nodes_rat_dag():
    """RAT-SPN DAG: region sums are shared by several products (no bias
    absorption there), multiple class roots."""
    g = rat_spn(13, F=16, D=2, R=2, S=3, I=4, C=3)
    x, _ = ancestral_sample(g, 1000, 14)
    _check(g, x)
    _check(g, nan_mask(x, 0.25, 15), marginal=True)


def test_tiny_discrete_normalisation_through_codegen():
    """Sum over all assignments of the generated code's joint = 1 (exactly
    normalised tiny discrete SPNs), and the all-missing marginal is log 1."""
    import itertools
    for seed in range(6):
        g = tiny_discrete_spn(seed)
        doms = g.meta["domains"]
        x = np.array(list(itertools.product(*[range(k) for k in doms])), np.float32)
        out, _, _ = host_eval(g, x, False)
        assert abs(np.exp(out[:, 0].astype(np.float64)).sum() - 1.0) < 1e-5
        allnan = np.full((4, len(doms)), np.nan, np.float32)
        m, _, _ = host_eval(g, allnan, True)
        assert np.abs(m).max() < 1e-5


def test_tiny_gaussian():
    for seed in range(4):
        g = tiny_gaussian_spn(seed)
        x = np.random.default_rng(seed).normal(0, 2, size=(300, g.n_features)).astype(np.float32)
        _check(g, x)
        _check(g, nan_mask(x, 0.4, seed), marginal=True)


def test_ptx_assembles_for_sm100a():
    for g, space in ((toy_spn(), 1), (toy_spn(), 2), (speaker_spn(2001), 0)):
        G = spnb.Graph(g)
        cg = spnb.codegen(G, 0, lang="ptx", compile=True, space=space)
        src = cg["source"]
        assert ".target sm_100a" in src and "lg2.approx.ftz.f32" in src
        assert ("ex2.approx.ftz.f32" in src) == (space != 2)
        assert cg["name"] + "_j" in src and cg["name"] + "_m" in src


# ---------------------------------------------------------------- value spaces (f4)
@pytest.mark.parametrize("space", [1, 2])
def test_codegen_value_spaces_discrete(space):
    """Log2 space and linear fp32 space give the oracle's values on the toy
    SPN (joint + marginal, out-of-support values) and on exhaustive inputs
    of tiny discrete SPNs (the `probability` type)."""
    g = toy_spn()
    x = toy_data(3000, seed=15)
    _check(g, x, False, space)
    _check(g, nan_mask(x, 0.3, 16), True, space)
    for seed in range(4):
        g = tiny_discrete_spn(seed)
        doms = g.meta["domains"]
        x = np.array(list(itertools.product(*[range(-1, k + 1) for k in doms])), np.float32)
        _check(g, x, False, space)
        _check(g, nan_mask(x, 0.3, seed), True, space)


def test_codegen_value_space_auto_rule():
    """Auto: linear for discrete SPNs inside the range bound (one lg2 per
    root, no ex2 in the generated code), log2 for Gaussian SPNs; forcing
    linear space on a Gaussian SPN is refused."""
    lin = spnb.codegen(spnb.Graph(toy_spn()), 0, lang="ptx")["source"]
    assert "ex2.approx" not in lin and lin.count("lg2.approx") == 2   # 1 root x (joint, marginal)
    log = spnb.codegen(spnb.Graph(toy_spn()), 0, lang="ptx", space=1)["source"]
    assert "ex2.approx" in log
    gauss = spnb.codegen(spnb.Graph(speaker_spn(2001)), 0, lang="ptx")["source"]
    assert "ex2.approx" in gauss
    with pytest.raises(spnb.SPNError):
        spnb.codegen(spnb.Graph(speaker_spn(2001)), 0, space=2)
