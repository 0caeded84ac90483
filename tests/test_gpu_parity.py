"""GPU parity: the sm_100a path (through the C ABI) against the fp64 oracle on
the same seeded inputs.  Tolerance (north_star): |g - o| <= 1e-4 max(1, |o|);
-inf must match -inf, NaN must match NaN.  Argmax must agree wherever the
oracle's top-2 gap exceeds twice the tolerance (ties are legitimately
decided by rounding)."""
import numpy as np
import pytest

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")

import paper_conf_cgo_sommera022_b200 as spnb  # noqa: E402
from oracle import oracle_eval  # noqa: E402
from spn_inputs import (toy_spn, speaker_spn, speaker_set, rat_spn, tiny_discrete_spn,  # noqa: E402
                        ancestral_sample, add_outliers, nan_mask, toy_data, GraphBuilder)

TOL = 1e-4


@pytest.fixture(scope="module", autouse=True)
def _lib():
    from paper_conf_cgo_sommera022_b200.build import build
    build()
    spnb.load_library()


def _cmp(gpu, ref, tol=TOL):
    gpu = np.asarray(gpu, dtype=np.float64)
    both_nan = np.isnan(gpu) & np.isnan(ref)
    both_inf = np.isneginf(gpu) & np.isneginf(ref)
    with np.errstate(invalid="ignore"):
        err = np.abs(gpu - ref) / np.maximum(1.0, np.abs(ref))
        ok = both_nan | both_inf | (err <= tol)
    assert ok.all(), (f"{(~ok).sum()} mismatches; first at {np.argwhere(~ok)[:3].tolist()}: "
                      f"gpu={gpu[~ok][:3]} ref={ref[~ok][:3]}")
    return float(np.nanmax(np.where(both_nan | both_inf, 0.0, err))) if err.size else 0.0


def _cmp_argmax(am_gpu, ref, am_ref, tol=TOL):
    if ref.shape[1] < 2:
        return
    s = np.sort(np.where(np.isnan(ref), -np.inf, ref), axis=1)
    gap = s[:, -1] - s[:, -2]
    decided = gap > 2 * tol * np.maximum(1.0, np.abs(s[:, -1]))
    assert np.array_equal(am_gpu[decided], am_ref[decided])


def _run(g, x, marginal=False, **opt):
    G = spnb.Graph(g)
    P = spnb.Plan(G, **opt)
    xt = torch.from_numpy(x).cuda()
    out, am = P.infer(xt, marginal=marginal)
    torch.cuda.synchronize()
    return out.cpu().numpy(), am.cpu().numpy(), P


def _parity(g, x, marginal=False, **opt):
    out, am, P = _run(g, x, marginal, **opt)
    ref, am_ref = oracle_eval(g, x, marginal=marginal)
    err = _cmp(out, ref)
    _cmp_argmax(am, ref, am_ref)
    return err, P


# ----------------------------------------------------------------- config 1
def test_c1_toy_all_assignments_and_golden():
    g = toy_spn()
    grid = np.array([[a, b, c] for a in range(-1, 3) for b in range(-1, 4) for c in range(-1, 5)],
                    np.float32)
    _parity(g, grid)
    pats = np.array([[a, b, c] for a in [np.nan, 0, 1] for b in [np.nan, 0, 1, 2]
                     for c in [np.nan, 0, 1, 2, 3]], np.float32)
    _parity(g, pats, marginal=True)


def test_c1_toy_100k_joint_and_marginal():
    g = toy_spn()
    x = toy_data(100_000, seed=1001)
    _parity(g, x)
    _parity(g, nan_mask(x, 0.2, 1002), marginal=True)


@pytest.mark.parametrize("space", [1, 2])
def test_value_space_selection(space):
    """f4: the toy and tiny discrete SPNs in log2 space and in
    linear fp32 space through the compiled path; auto picks linear for them
    and log2 for Gaussian SPNs; linear is refused for a Gaussian SPN."""
    import itertools
    g = toy_spn()
    x = toy_data(200_000, seed=1003)
    err, P = _parity(g, x, value_space=space)
    assert P.info()["path"] == 2 and P.info()["value_space"] == space
    _parity(g, nan_mask(x, 0.2, 1004), marginal=True, value_space=space)
    for seed in range(3):
        gd = tiny_discrete_spn(seed)
        doms = gd.meta["domains"]
        xd = np.array(list(itertools.product(*[range(-1, k + 1) for k in doms])), np.float32)
        _parity(gd, xd, value_space=space)
        _parity(gd, nan_mask(xd, 0.3, seed), marginal=True, value_space=space)
    if space == 2:
        assert spnb.Plan(spnb.Graph(toy_spn())).info()["value_space"] == 2       # auto
        assert spnb.Plan(spnb.Graph(speaker_spn(2001))).info()["value_space"] == 1
        with pytest.raises(spnb.SPNError):
            spnb.Plan(spnb.Graph(speaker_spn(2001)), value_space=2)


# ----------------------------------------------------------------- config 2
@pytest.mark.parametrize("n", [1, 31, 128, 129, 1000, 4099])
def test_c2_ragged_sizes(n):
    g = speaker_spn(2001)
    x, _ = ancestral_sample(g, n, 2002)
    _parity(g, add_outliers(x, 0.01, 7))


@pytest.mark.parametrize("K", [1, 2, 4])
def test_c2_samples_per_thread_variants(K):
    g = speaker_spn(2001)
    x, _ = ancestral_sample(g, 3000, 11)
    _parity(g, add_outliers(x, 0.01, 7), samples_per_thread=K)


def test_c2_full_size_sampled():
    """1M samples in the bench's launch configuration; oracle on a sample."""
    g = speaker_spn(2001)
    x, _ = ancestral_sample(g, 1_000_000, 2002)
    x = add_outliers(x, 0.01, 2003)
    out, _, P = _run(g, x)
    idx = np.random.default_rng(0).choice(len(x), 4000, replace=False)
    ref, _ = oracle_eval(g, x[idx])
    _cmp(out[idx], ref)
    assert np.isfinite(out).all()


def test_c2_marginal_without_nan_is_bitwise_joint():
    g = speaker_spn(2001)
    x, _ = ancestral_sample(g, 5000, 3)
    G = spnb.Graph(g)
    P = spnb.Plan(G)
    xt = torch.from_numpy(x).cuda()
    j, _ = P.infer(xt)
    m, _ = P.infer(xt, marginal=True)
    assert torch.equal(j, m)


def test_c2_full_marginal_is_zero():
    g = speaker_spn(2001)
    x = np.full((257, 26), np.nan, np.float32)
    out, _, _ = _run(g, x, marginal=True)
    assert np.abs(out).max() < 1e-4


# ----------------------------------------------------------------- config 3
def test_c3_speaker_set_marginal_argmax():
    g = speaker_set(list(range(3001, 3033)))
    x, labels = ancestral_sample(g, 3000, 3002)
    x = nan_mask(x, 0.2, 3100)
    err, P = _parity(g, x, marginal=True)
    assert P.info()["n_tasks"] >= 1


def test_c3_partition_sizes_agree():
    g = speaker_set(list(range(3001, 3009)))
    x, _ = ancestral_sample(g, 2000, 5)
    x = nan_mask(x, 0.2, 6)
    outs = []
    for cap in (0, 300, 2000):
        out, am, P = _run(g, x, True, max_task_nodes=cap)
        outs.append(out)
        ref, am_ref = oracle_eval(g, x, marginal=True)
        _cmp(out, ref)
    for o in outs[1:]:
        _cmp(o, outs[0].astype(np.float64), tol=1e-5)


# ----------------------------------------------------------------- config 4 (generic path)
def test_c4_rat_generic_path_small():
    g = rat_spn(4001, F=784, D=5, R=2, S=8, I=10, C=10)
    x, _ = ancestral_sample(g, 600, 4002)
    _parity(g, x)


def test_rat_generic_with_partitioning():
    g = rat_spn(7, F=64, D=3, R=3, S=6, I=8, C=4)
    x, _ = ancestral_sample(g, 700, 8)
    for cap in (0, 500):
        _parity(g, x, max_task_nodes=cap)


# ----------------------------------------------------------------- edges
def test_empty_batch_and_strided_input():
    g = speaker_spn(2001)
    G = spnb.Graph(g)
    P = spnb.Plan(G)
    x, _ = ancestral_sample(g, 500, 1)
    big = torch.zeros((500, 40), dtype=torch.float32, device="cuda")
    big[:, :26] = torch.from_numpy(x).cuda()
    out, _ = P.infer(big)                       # ld = 40 > F
    ref, _ = oracle_eval(g, x)
    _cmp(out.cpu().numpy(), ref)
    e, _ = P.infer(big[:0])                     # n = 0 no-op
    assert e.shape == (0, 1)
    with pytest.raises(ValueError):
        P.infer(big[:, :20])                    # fewer columns than features
    lib = spnb.load_library()
    import ctypes
    rc = lib.spn_infer_joint(P._h, ctypes.c_void_p(big.data_ptr()), 10, 20,
                             ctypes.c_void_p(out.data_ptr()), None, None)
    assert rc == -1                             # SPN_E_ARG: ld < n_features


def test_shard_invariance_bitwise():
    g = speaker_set(list(range(3001, 3005)))
    x, _ = ancestral_sample(g, 10_000, 2)
    G = spnb.Graph(g)
    P = spnb.Plan(G)
    xt = torch.from_numpy(x).cuda()
    full, amf = P.infer(xt)
    parts = [P.infer(xt[a:b]) for a, b in ((0, 3333), (3333, 7001), (7001, 10_000))]
    assert torch.equal(full, torch.cat([p[0] for p in parts]))
    assert torch.equal(amf, torch.cat([p[1] for p in parts]))


def test_host_pipeline_matches_device():
    g = speaker_spn(2001)
    x, _ = ancestral_sample(g, 300_000, 5)
    G = spnb.Graph(g)
    P = spnb.Plan(G)
    dev, _ = P.infer(torch.from_numpy(x).cuda())
    xh = torch.from_numpy(x).pin_memory()
    out, am = P.infer_host(xh)
    assert np.array_equal(out, dev.cpu().numpy())


def test_tiny_discrete_exact():
    import itertools
    for seed in range(4):
        g = tiny_discrete_spn(seed)
        doms = g.meta["domains"]
        x = np.array(list(itertools.product(*[range(-1, k + 1) for k in doms])), np.float32)
        _parity(g, x)
        _parity(g, nan_mask(x, 0.3, seed), marginal=True)


# ----------------------------------------------------------------- layered tensor-core path (a5)
@pytest.mark.parametrize("kernel", [1, 2])
@pytest.mark.parametrize("shape", [(32, 2, 2, 4, 8, 3), (64, 3, 3, 8, 16, 5), (24, 1, 1, 4, 8, 2),
                                   (128, 3, 2, 20, 40, 10)])
def test_layered_rat_small_matches_oracle(shape, kernel):
    """Both layered kernels (v1 rat_eval.cu, v2 rat2.cu), hi/lo and single
    f16 passes, joint and marginal."""
    F, D, R, S, I, C = shape
    g = rat_spn(11, F=F, D=D, R=R, S=S, I=I, C=C)
    x, _ = ancestral_sample(g, 1000, 12)
    # v2: certified with tensor-core leaves (leaf_tc 2), certified with FMA
    # leaves (auto), raw single pass (FMA leaves); v1: hi/lo
    for prec, ltc in (((0, 2), (0, 0), (1, 0)) if kernel == 2 else ((2, 0),)):
        err, P = _parity(g, x, layered_path=2, tc_precision=prec, layered_kernel=kernel, leaf_tc=ltc)
        info = P.info()
        assert info["path"] == 1 and info["layered_kernel"] == kernel
        assert info["leaf_tc"] == (1 if ltc == 2 else 0)
        _parity(g, nan_mask(x, 0.2, 13), marginal=True, layered_path=2, tc_precision=prec,
                layered_kernel=kernel, leaf_tc=ltc)


@pytest.mark.parametrize("shape", [(32, 2, 2, 4, 8, 3), (128, 3, 2, 20, 40, 10)])
def test_layered_leaf_tc_out_of_range_inputs(shape):
    """Tensor-core leaves: inputs outside the f16 split's range (|x - M| > 240,
    +-inf) and NaN in a joint query are recomputed by the certification
    (v1, FMA leaves); every row matches the oracle (NaN / -inf included)."""
    F, D, R, S, I, C = shape
    g = rat_spn(15, F=F, D=D, R=R, S=S, I=I, C=C)
    x, _ = ancestral_sample(g, 3000, 16)
    rng = np.random.default_rng(17)
    rows = rng.choice(len(x), 60, replace=False)
    cols = rng.integers(0, F, size=60)
    vals = np.array([1e3, -5e2, 300.0, np.inf, -np.inf, np.nan] * 10, dtype=np.float32)
    x[rows, cols] = vals
    err, P = _parity(g, x, layered_path=2, layered_kernel=2, leaf_tc=2)
    assert P.info()["leaf_tc"] == 1
    xm = nan_mask(x, 0.2, 18)
    _parity(g, xm, marginal=True, layered_path=2, layered_kernel=2, leaf_tc=2)


def test_layered_matches_generic_path():
    g = rat_spn(21, F=96, D=3, R=3, S=8, I=8, C=4)
    x, _ = ancestral_sample(g, 2000, 22)
    a, am_a, Pa = _run(g, x, layered_path=2, tc_precision=2)
    b, am_b, Pb = _run(g, x, layered_path=1)
    assert Pa.info()["path"] == 1 and Pb.info()["path"] == 0
    _cmp(a, b.astype(np.float64), tol=1e-5)


def test_c4_layered_full_graph_sampled():
    """Config 4 graph (518,730 nodes) on the layered path; oracle on a sample."""
    from spn_inputs import config_graph
    g = config_graph("C4")
    x, _ = ancestral_sample(g, 3000, 4002)
    for prec in (2, 1):
        out, am, P = _run(g, x, layered_path=2, tc_precision=prec)
        assert P.info()["path"] == 1
        idx = np.random.default_rng(0).choice(len(x), 300, replace=False)
        ref, am_ref = oracle_eval(g, x[idx])
        _cmp(out[idx], ref)
        _cmp_argmax(am[idx], ref, am_ref)


def test_layered_ragged_and_chunked():
    g = rat_spn(31, F=256, D=3, R=2, S=8, I=8, C=3)
    x = np.random.default_rng(32).uniform(0, 1, size=(80_001, 256)).astype(np.float32)
    out, am, P = _run(g, x, layered_path=2)     # > one transposed chunk, ragged tail
    assert P.info()["layered_kernel"] == 1      # (I, S) = (8, 8): no v2 instance
    idx = np.concatenate([np.arange(0, 50), np.arange(37_850, 37_950), np.arange(79_950, 80_001)])
    ref, _ = oracle_eval(g, x[idx])
    _cmp(out[idx], ref)


def test_layered_v2_ragged_and_chunked():
    """v2 kernel over two transposed chunks (148 x 128 x 8 samples each) with
    a ragged tail; rows from both chunk edges against the oracle."""
    g = rat_spn(33, F=128, D=3, R=2, S=4, I=8, C=3)
    x = np.random.default_rng(34).uniform(0, 1, size=(160_001, 128)).astype(np.float32)
    out, am, P = _run(g, x, layered_path=2)
    info = P.info()
    assert info["layered_kernel"] == 2 and info["chunk_samples"] < len(x)
    c = info["chunk_samples"]
    idx = np.concatenate([np.arange(0, 64), np.arange(c - 64, c + 64), np.arange(len(x) - 65, len(x))])
    ref, am_ref = oracle_eval(g, x[idx])
    _cmp(out[idx], ref)
    _cmp_argmax(am[idx], ref, am_ref)


# ----------------------------------------------------------------- compiled path (KS)
def test_compiled_path_is_default_for_speaker_spn():
    g = speaker_spn(2001)
    x, _ = ancestral_sample(g, 20_000, 41)
    x = add_outliers(x, 0.01, 42)
    err, P = _parity(g, x)
    info = P.info()
    assert info["path"] == 2 and info["n_tasks"] == 1, info
    _parity(g, nan_mask(x, 0.2, 43), marginal=True)


def test_compiled_matches_interpreter():
    g = speaker_spn(2002)
    x, _ = ancestral_sample(g, 10_000, 44)
    a, _, Pa = _run(g, x, compiled_path=2)
    b, _, Pb = _run(g, x, compiled_path=1)
    assert Pa.info()["path"] == 2 and Pb.info()["path"] == 0
    _cmp(a, b.astype(np.float64), tol=2e-6)


def test_compiled_multi_task_argmax():
    g = speaker_set(list(range(3001, 3009)))          # 8 components -> several tasks
    x, _ = ancestral_sample(g, 5000, 45)
    err, P = _parity(g, nan_mask(x, 0.2, 46), marginal=True, compiled_path=2)
    assert P.info()["path"] == 2 and P.info()["n_tasks"] > 1


def test_compiled_edge_values():
    g = speaker_spn(2001)
    x, _ = ancestral_sample(g, 512, 47)
    x[0, 3] = np.inf
    x[1, 5] = -np.inf
    x[2, 7] = np.nan
    x[3, :] = np.nan
    x[4, 1] = 1e15
    for marginal in (False, True):
        _parity(g, x, marginal=marginal, compiled_path=2)


@pytest.mark.parametrize("n", [1, 31, 255, 257, 100_003])
def test_compiled_ragged(n):
    g = toy_spn()
    x = toy_data(n, seed=n)
    _parity(g, x, compiled_path=2)
    _parity(g, nan_mask(x, 0.3, n), marginal=True, compiled_path=2)


def test_compiled_auto_skips_region_graphs():
    """Auto selection keeps RAT-SPN cross products (hundreds of live values)
    off the compiled path: prepare stays fast and the interpreter serves the
    graph (regression: ptxas took minutes on this graph)."""
    import time
    g = rat_spn(21, F=96, D=3, R=3, S=8, I=8, C=4)
    x, _ = ancestral_sample(g, 500, 23)
    t = time.perf_counter()
    err, P = _parity(g, x, layered_path=1)
    assert P.info()["path"] == 0
    assert time.perf_counter() - t < 60


def test_compiled_spill_fallback_marginal_full_size():
    """Config-2 graph, marginal kernel: launched without register spills
    (per-variant launch bounds), parity on a sample of a 1M-sample batch."""
    from spn_inputs import config_graph
    g = config_graph("C2")
    x, _ = ancestral_sample(g, 1_000_000, 2002)
    x = nan_mask(x, 0.2, 48)
    out, _, P = _run(g, x, marginal=True)
    assert P.info()["path"] == 2
    idx = np.random.default_rng(1).choice(len(x), 2000, replace=False)
    ref, _ = oracle_eval(g, x[idx], marginal=True)
    _cmp(out[idx], ref)


def test_c3_full_size_sampled():
    """Config 3 at its bench size (32 speaker SPNs, 1M samples, 20% NaN,
    marginal + argmax) in the bench's launch configuration; oracle on a
    sample of rows spread over the batch."""
    from spn_inputs import config_graph
    g = config_graph("C3")
    x, _ = ancestral_sample(g, 1_000_000, 3002)
    x = nan_mask(x, 0.2, 3100)
    out, am, P = _run(g, x, marginal=True)
    assert P.info()["path"] == 2
    idx = np.concatenate([np.arange(0, 200), np.random.default_rng(5).choice(len(x), 1500, replace=False),
                          np.arange(len(x) - 200, len(x))])
    ref, am_ref = oracle_eval(g, x[idx], marginal=True)
    _cmp(out[idx], ref)
    _cmp_argmax(am[idx], ref, am_ref)


def test_c4_layered_marginal_full_graph_sampled():
    """Config 4 graph on the layered path with 20% missing features."""
    from spn_inputs import config_graph
    g = config_graph("C4")
    x, _ = ancestral_sample(g, 2000, 4003)
    x = nan_mask(x, 0.2, 4004)
    out, am, P = _run(g, x, marginal=True, layered_path=2)
    assert P.info()["path"] == 1
    idx = np.random.default_rng(6).choice(len(x), 200, replace=False)
    ref, am_ref = oracle_eval(g, x[idx], marginal=True)
    _cmp(out[idx], ref)
    _cmp_argmax(am[idx], ref, am_ref)


def test_c5_layered_full_graph_sampled():
    """Config 5 graph (3,242,010 nodes) on the layered path in the bench's
    launch configuration (default plan, counter-based U[0,1] inputs) over two
    transposed chunks with a ragged tail; oracle on rows from the start, the
    chunk boundary and the end."""
    from spn_inputs import config_graph, uniform_chunked
    g = config_graph("C5")
    G = spnb.Graph(g)
    P = spnb.Plan(G)
    c = P.info()["chunk_samples"]
    n = c + 10_001
    x = uniform_chunked(n, g.n_features, 5002)
    out, am = P.infer(torch.from_numpy(x).cuda())
    torch.cuda.synchronize()
    out, am = out.cpu().numpy(), am.cpu().numpy()
    assert P.info()["path"] == 1 and P.info()["layered_kernel"] == 2
    idx = np.concatenate([np.arange(0, 16), np.arange(c - 16, c + 16), np.arange(n - 16, n)])
    ref, am_ref = oracle_eval(g, x[idx])
    _cmp(out[idx], ref)
    _cmp_argmax(am[idx], ref, am_ref)


def test_c5_layered_marginal_sampled():
    """Config 5 graph on the layered path (default plan: certified single
    f16 pass) with 20% missing features: marginal query on ancestral samples
    and on the bench's U[0,1] inputs, oracle on rows of both."""
    from spn_inputs import config_graph, uniform_chunked
    g = config_graph("C5")
    P = spnb.Plan(spnb.Graph(g))
    assert P.info()["path"] == 1 and P.info()["layered_kernel"] == 2
    xa, _ = ancestral_sample(g, 4000, 5005)
    xu = uniform_chunked(20_000, g.n_features, 5006)
    for x, seed in ((xa, 5007), (xu, 5008)):
        x = nan_mask(x, 0.2, seed)
        out, am = P.infer(torch.from_numpy(x).cuda(), marginal=True)
        torch.cuda.synchronize()
        out, am = out.cpu().numpy(), am.cpu().numpy()
        idx = np.random.default_rng(seed).choice(len(x), 24, replace=False)
        ref, am_ref = oracle_eval(g, x[idx], marginal=True)
        _cmp(out[idx], ref)
        _cmp_argmax(am[idx], ref, am_ref)


def test_c5_partitioned_generic_vs_layered_vs_oracle():
    """BASELINE configs[4] "partitioned into tasks": the C5 graph through the
    generic interpreter with the paper's <= 10k-operation tasks (PAPER.md
    L336-346, L481-485; several thousand tasks, cut values in global
    scratch) on 10k ancestral samples, against the layered tensor-core path
    on all 10k rows and both against the fp64 oracle on 1k rows."""
    from spn_inputs import config_graph
    g = config_graph("C5")
    x, _ = ancestral_sample(g, 10_000, 5003)
    G = spnb.Graph(g)
    Pg = spnb.Plan(G, layered_path=1, compiled_path=1, max_task_nodes=10_000)
    ig = Pg.info()
    assert ig["path"] == 0 and ig["n_tasks"] > 1000 and ig["n_global_slots"] > 0, ig
    xt = torch.from_numpy(x).cuda()
    og, amg = Pg.infer(xt)
    Pl = spnb.Plan(G)
    assert Pl.info()["path"] == 1
    ol, aml = Pl.infer(xt)
    torch.cuda.synchronize()
    og, amg, ol, aml = og.cpu().numpy(), amg.cpu().numpy(), ol.cpu().numpy(), aml.cpu().numpy()
    _cmp(og, ol.astype(np.float64))
    idx = np.random.default_rng(7).choice(len(x), 1000, replace=False)
    ref, am_ref = oracle_eval(g, x[idx])
    _cmp(og[idx], ref)
    _cmp(ol[idx], ref)
    _cmp_argmax(amg[idx], ref, am_ref)
    _cmp_argmax(aml[idx], ref, am_ref)


@pytest.mark.parametrize("which", ["compiled", "interpreter", "layered"])
def test_host_api_matches_oracle(which):
    """spn_infer_*_host (pinned host buffers, chunked copies overlapped with
    compute on two streams) over more than two host
    chunks: bitwise equal to the device-buffer call and within tolerance of
    the oracle on rows from every chunk."""
    from spn_inputs import config_graph
    if which == "compiled":
        g, n, opt = speaker_spn(2001), 2_600_000, {}
    elif which == "interpreter":
        g, n, opt = rat_spn(41, F=256, D=3, R=3, S=6, I=8, C=4), 70_000, {"layered_path": 1,
                                                                           "compiled_path": 1,
                                                                           "max_task_nodes": 400}
    else:
        g, n, opt = config_graph("C4"), 20_000, {}
    x, _ = ancestral_sample(g, n, 42)
    G = spnb.Graph(g)
    P = spnb.Plan(G, **opt)
    dev, amd = P.infer(torch.from_numpy(x).cuda())
    xh = torch.from_numpy(x).pin_memory()
    out, am = P.infer_host(xh)
    assert np.array_equal(out, dev.cpu().numpy())
    assert np.array_equal(am, amd.cpu().numpy())
    idx = np.linspace(0, n - 1, 240).astype(np.int64)
    ref, am_ref = oracle_eval(g, x[idx])
    _cmp(out[idx], ref)
    _cmp_argmax(am[idx], ref, am_ref)


def test_host_api_layered_certified_groups(monkeypatch):
    """Certified layered plans pipeline host rows group-wise (one
    certification round per group, api.cpp infer_host_grouped): several
    groups of one transposed chunk each plus a ragged tail, joint and
    marginal, bitwise equal to the device-buffer call and within tolerance
    of the oracle on rows of every group."""
    from spn_inputs import config_graph, uniform_chunked
    monkeypatch.setenv("SPNB_HOST_GROUP_CHUNKS", "1")
    g = config_graph("C4")
    G = spnb.Graph(g)
    P = spnb.Plan(G)
    info = P.info()
    assert info["path"] == 1 and info["layered_kernel"] == 2 and info["certified"] == 1
    c = info["chunk_samples"]
    n = 2 * c + 7_777
    x = uniform_chunked(n, g.n_features, 4242)   # the bench's inputs: mostly certified
    x[::997] = ancestral_sample(g, len(x[::997]), 4243)[0]  # some rows the v1 recompute serves
    x[::97, 5] = np.nan
    xh = torch.from_numpy(x).pin_memory()
    # a small call first (buffers sized for it), then the full call regrows them
    small, _ = P.infer_host(torch.from_numpy(x[:1000]).pin_memory())
    for marginal in (False, True):
        dev, amd = P.infer(torch.from_numpy(x).cuda(), marginal=marginal)
        out, am = P.infer_host(xh, marginal=marginal)
        if not marginal:
            assert np.array_equal(small, out[:1000], equal_nan=True)
        assert np.array_equal(out, dev.cpu().numpy(), equal_nan=True)
        assert np.array_equal(am, amd.cpu().numpy())
        idx = np.concatenate([np.arange(0, 8), np.arange(c - 4, c + 4), np.arange(2 * c - 4, 2 * c + 4),
                              np.arange(n - 8, n)])
        ref, am_ref = oracle_eval(g, x[idx], marginal=marginal)
        _cmp(out[idx], ref)
        _cmp_argmax(am[idx], ref, am_ref)
