"""Pins for the fp64 oracle (task rule ③): every oracle function is checked
against something other than itself -- hand-computed exact values, exact
rational arithmetic, textbook/library routines (scipy / sklearn), closed forms,
brute force over all assignments, and quadrature.  CPU only."""
import itertools
import math
import os

import numpy as np
import pytest
from scipy import integrate, special, stats

from oracle import oracle_eval
from oracle.exact import exact_probability, exact_log
from spn_inputs import (GraphBuilder, toy_spn, tiny_discrete_spn, tiny_gaussian_spn,
                        speaker_spn, rat_spn, rat_counts, ancestral_sample)

GOLDEN = os.path.join(os.path.dirname(__file__), "golden", "toy_appendixA.txt")


def _read_golden():
    rows = []
    for line in open(GOLDEN):
        line = line.strip()
        if not line or line.startswith("#"):
            continue
        a, b, c, frac, lnp = line.split()
        xs = [float("nan") if t == "nan" else float(t) for t in (a, b, c)]
        num, den = frac.split("/")
        rows.append((xs, int(num), int(den), float(lnp)))
    return rows


# ---------------------------------------------------------------- toy (C1)
def test_toy_exact_matches_hand_computed_golden():
    from fractions import Fraction
    g = toy_spn()
    for xs, num, den, _ in _read_golden():
        (p,) = exact_probability(g, xs, marginal=True)
        assert p == Fraction(num, den), (xs, p)


def test_toy_c_oracle_matches_golden():
    g = toy_spn()
    rows = _read_golden()
    x = np.array([r[0] for r in rows], dtype=np.float32)
    lp, _ = oracle_eval(g, x, marginal=True)
    for (xs, num, den, lnp), v in zip(rows, lp[:, 0]):
        if math.isinf(lnp):
            assert v == -np.inf
        else:
            assert abs(v - lnp) <= 1e-12, (xs, v, lnp)


def test_toy_normalisation_and_all_marginal_patterns():
    """All 24 joint assignments sum to exactly 1; each of the 60 partial
    evidence patterns equals the exact sum of the joint over the missing
    variables (marginal inference definition)."""
    from fractions import Fraction
    g = toy_spn()
    doms = [2, 3, 4]
    joint = {}
    for a in itertools.product(*[range(k) for k in doms]):
        joint[a] = exact_probability(g, [float(v) for v in a])[0]
    assert sum(joint.values()) == Fraction(1)
    pats = list(itertools.product(*[[None] + list(range(k)) for k in doms]))
    assert len(pats) == 60
    xs = np.array([[np.nan if v is None else float(v) for v in p] for p in pats], np.float32)
    lp, _ = oracle_eval(g, xs, marginal=True)
    for p, v in zip(pats, lp[:, 0]):
        tot = sum(pr for a, pr in joint.items()
                  if all(pi is None or pi == ai for pi, ai in zip(p, a)))
        assert exact_probability(g, [np.nan if t is None else float(t) for t in p])[0] == tot
        ref = exact_log(tot)
        if ref == -math.inf:
            assert v == -np.inf
        else:
            assert abs(v - ref) <= 1e-12


def test_toy_c_oracle_joint_all_assignments_match_fractions():
    g = toy_spn()
    xs = np.array(list(itertools.product(range(-1, 3), range(-1, 4), range(-1, 5))), np.float32)
    lp, _ = oracle_eval(g, xs, marginal=False)
    for x, v in zip(xs, lp[:, 0]):
        ref = exact_log(exact_probability(g, list(x))[0])
        assert (v == ref) if ref == -math.inf else abs(v - ref) < 1e-12


# ------------------------------------------------- tiny discrete (B3) brute force
@pytest.mark.parametrize("seed", range(12))
def test_tiny_discrete_normalises_and_marginalises(seed):
    g = tiny_discrete_spn(seed, n_vars=3 + seed % 2)
    doms = g.meta["domains"]
    allx = np.array(list(itertools.product(*[range(k) for k in doms])), np.float32)
    lp, _ = oracle_eval(g, allx, marginal=False)
    assert abs(special.logsumexp(lp[:, 0])) < 1e-12          # sum over all = 1
    # every single-variable-missing pattern equals log-sum of the joint
    rng = np.random.default_rng(seed)
    for _ in range(6):
        a = [int(rng.integers(0, k)) for k in doms]
        miss = int(rng.integers(0, len(doms)))
        q = np.array([[np.nan if i == miss else a[i] for i in range(len(doms))]], np.float32)
        mv, _ = oracle_eval(g, q, marginal=True)
        comp = np.array([[v if i != miss else t for i, v in enumerate(a)]
                         for t in range(doms[miss])], np.float32)
        jv, _ = oracle_eval(g, comp, marginal=False)
        assert abs(mv[0, 0] - special.logsumexp(jv[:, 0])) < 1e-12
        # and equals the exact rational marginal
        assert abs(mv[0, 0] - exact_log(exact_probability(g, list(q[0]))[0])) < 1e-12
    # everything missing -> log 1 = 0
    z, _ = oracle_eval(g, np.full((1, len(doms)), np.nan, np.float32), marginal=True)
    assert abs(z[0, 0]) < 1e-14


# ------------------------------------------------------------- leaves
def test_gaussian_leaf_matches_scipy_logpdf():
    rng = np.random.default_rng(0)
    for _ in range(20):
        mu, sd = rng.normal() * 3, rng.uniform(0.05, 4)
        b = GraphBuilder(1)
        r = b.gaussian(0, mu, sd)
        g = b.build([r])
        x = rng.normal(mu, 3 * sd, size=(50, 1)).astype(np.float32)
        lp, _ = oracle_eval(g, x)
        ref = stats.norm.logpdf(x[:, 0].astype(np.float64), loc=mu, scale=sd)
        np.testing.assert_allclose(lp[:, 0], ref, rtol=1e-13, atol=1e-12)


def test_categorical_and_histogram_leaves():
    b = GraphBuilder(2)
    c = b.categorical(0, [0.1, 0.6, 0.3])
    h = b.histogram(1, [(-2, 0, 0.05), (0, 3, 0.1), (5, 6, 0.3)])
    g = b.build([c, h])
    xs = np.array([[0, -2], [0.99, -0.5], [1, 0], [2.5, 2.999], [3, 3], [-0.01, 4],
                   [2, 5.5], [-1, 6], [np.inf, -np.inf]], np.float32)
    lp, _ = oracle_eval(g, xs)
    exp_c = [math.log(.1), math.log(.1), math.log(.6), math.log(.3), -math.inf,
             -math.inf, math.log(.3), -math.inf, -math.inf]
    exp_h = [math.log(.05), math.log(.05), math.log(.1), math.log(.1), -math.inf,
             -math.inf, math.log(.3), -math.inf, -math.inf]
    for v, e in zip(lp[:, 0], exp_c):
        assert v == e or abs(v - e) < 1e-15
    for v, e in zip(lp[:, 1], exp_h):
        assert v == e or abs(v - e) < 1e-15


def test_nan_semantics_joint_vs_marginal():
    """Reading c7: a joint query propagates NaN; reading c6: marginal -> log 1."""
    b = GraphBuilder(2)
    g0 = b.gaussian(0, 0.0, 1.0)
    c1 = b.categorical(1, [0.5, 0.5])
    p = b.product([g0, c1])
    s = b.sum([p, b.product([b.gaussian(0, 1.0, 2.0), b.categorical(1, [0.2, 0.8])])], [0.4, 0.6])
    g = b.build([s, g0, c1])
    x = np.array([[np.nan, 1.0], [0.3, np.nan], [np.nan, np.nan]], np.float32)
    j, _ = oracle_eval(g, x, marginal=False)
    assert np.array_equal(np.isnan(j), [[True, True, False], [True, False, True],
                                        [True, True, True]])
    m, am = oracle_eval(g, x, marginal=True)
    assert m[2, 0] == pytest.approx(0.0, abs=1e-15)
    assert m[0, 1] == 0.0 and m[1, 2] == 0.0
    x3 = float(np.float32(0.3))
    ref = special.logsumexp([stats.norm.logpdf(x3, 0, 1), stats.norm.logpdf(x3, 1, 2)],
                            b=[0.4, 0.6])
    assert m[1, 0] == pytest.approx(ref, abs=1e-13)


# ------------------------------------------------------------- inner nodes
def test_sum_node_matches_scipy_logsumexp():
    rng = np.random.default_rng(1)
    for n in (1, 2, 3, 7, 40):
        b = GraphBuilder(1)
        mus, sds = rng.normal(size=n), rng.uniform(0.2, 2, size=n)
        w = rng.dirichlet(np.ones(n)) * rng.uniform(0.5, 2)   # not normalised (c9)
        leaves = [b.gaussian(0, m, s) for m, s in zip(mus, sds)]
        g = b.build([b.sum(leaves, w)])
        x = rng.normal(0, 4, size=(30, 1)).astype(np.float32)
        lp, _ = oracle_eval(g, x)
        comp = stats.norm.logpdf(x.astype(np.float64), loc=mus[None], scale=sds[None])
        ref = special.logsumexp(comp, b=w[None], axis=1)
        np.testing.assert_allclose(lp[:, 0], ref, rtol=1e-13, atol=1e-12)


def test_sum_with_zero_weights_and_all_minus_inf():
    b = GraphBuilder(1)
    c = b.categorical(0, [1.0, 0.0])
    d = b.categorical(0, [0.0, 1.0])
    g = b.build([b.sum([c, d], [1.0, 0.0])])
    lp, _ = oracle_eval(g, np.array([[0], [1], [5]], np.float32))
    assert lp[0, 0] == 0.0 and lp[1, 0] == -np.inf and lp[2, 0] == -np.inf


def test_product_is_sum_of_logpdfs():
    rng = np.random.default_rng(2)
    F = 9
    b = GraphBuilder(F)
    mus, sds = rng.normal(size=F), rng.uniform(0.3, 2, size=F)
    g = b.build([b.product([b.gaussian(f, mus[f], sds[f]) for f in range(F)])])
    x = rng.normal(size=(40, F)).astype(np.float32)
    lp, _ = oracle_eval(g, x)
    ref = stats.norm.logpdf(x.astype(np.float64), mus[None], sds[None]).sum(1)
    np.testing.assert_allclose(lp[:, 0], ref, rtol=1e-13, atol=1e-11)


def test_diagonal_gmm_matches_sklearn():
    """Root sum over K products of F Gaussians == diag-covariance GMM."""
    from sklearn.mixture import GaussianMixture
    rng = np.random.default_rng(3)
    K, F = 5, 6
    w = rng.dirichlet(np.ones(K))
    mu = rng.normal(size=(K, F)) * 2
    sd = rng.uniform(0.3, 1.5, size=(K, F))
    b = GraphBuilder(F)
    prods = [b.product([b.gaussian(f, mu[k, f], sd[k, f]) for f in range(F)]) for k in range(K)]
    g = b.build([b.sum(prods, w)])
    gm = GaussianMixture(n_components=K, covariance_type="diag")
    gm.weights_ = w
    gm.means_ = mu
    gm.covariances_ = sd ** 2
    gm.precisions_cholesky_ = 1.0 / sd
    x = rng.normal(size=(200, F)).astype(np.float32) * 2
    lp, _ = oracle_eval(g, x)
    np.testing.assert_allclose(lp[:, 0], gm.score_samples(x.astype(np.float64)),
                               rtol=1e-12, atol=1e-11)


@pytest.mark.parametrize("seed", [0, 1, 2])
def test_gaussian_marginal_matches_quadrature(seed):
    g = tiny_gaussian_spn(seed, n_vars=2)
    for x0 in (-1.3, 0.2, 1.7):
        m, _ = oracle_eval(g, np.array([[x0, np.nan]], np.float32), marginal=True)
        f = lambda t: math.exp(oracle_eval(g, np.array([[x0, t]], np.float32),
                                           want_argmax=False)[0][0, 0])
        # the float32 cast of t is harmless: the integrand is smooth
        val, _ = integrate.quad(f, -30, 30, limit=400, epsabs=1e-13)
        assert abs(m[0, 0] - math.log(val)) < 1e-6


def test_full_marginal_is_zero_and_no_nan_marginal_equals_joint():
    g = speaker_spn(2001)
    z, _ = oracle_eval(g, np.full((3, 26), np.nan, np.float32), marginal=True)
    assert np.all(np.abs(z) < 1e-12)
    x, _ = ancestral_sample(g, 500, 7)
    j, _ = oracle_eval(g, x, marginal=False)
    m, _ = oracle_eval(g, x, marginal=True)
    assert np.array_equal(j, m)


def test_argmax_lowest_index_ties_and_nan():
    b = GraphBuilder(1)
    c0 = b.categorical(0, [0.5, 0.5])
    c1 = b.categorical(0, [0.5, 0.5])
    c2 = b.categorical(0, [0.25, 0.75])
    g = b.build([c0, c1, c2])
    lp, am = oracle_eval(g, np.array([[0], [1], [7], [np.nan]], np.float32))
    assert list(am) == [0, 2, 0, -1]


# ---------------------------------------------------------- RAT-SPN structure
def test_rat_counts_match_closed_form():
    g = rat_spn(11, F=64, D=3, R=2, S=4, I=5, C=3)
    c = g.counts()
    ref = rat_counts(64, 3, 2, 4, 5, 3)
    assert c["gaussian"] == ref["leaves"] and c["product"] == ref["products"]
    assert c["sum"] == ref["sums"] and c["nodes"] == ref["nodes"]
    assert rat_counts(784, 5, 8, 20, 40, 10)["nodes"] == 518_730
    assert rat_counts(784, 5, 50, 20, 40, 10)["nodes"] == 3_242_010


def test_rat_depth1_is_closed_form_mixture():
    """A RAT-SPN with D=1, R=1 is a diagonal mixture with I^2 components:
    log p_c = logsumexp_{ij} (log W_c[i,j] + log A_i(x) + log B_j(x))."""
    F, I, C = 10, 4, 3
    g = rat_spn(5, F=F, D=1, R=1, S=3, I=I, C=C)
    rat = g.meta["rat"]
    (la, lb) = rat["reps"][0]["leaves"]
    x = np.random.default_rng(9).uniform(-0.5, 1.5, size=(50, F)).astype(np.float32)
    xd = x.astype(np.float64)
    A = stats.norm.logpdf(xd[:, None, la["vars"]], la["mu"][None], la["sd"][None]).sum(-1)
    B = stats.norm.logpdf(xd[:, None, lb["vars"]], lb["mu"][None], lb["sd"][None]).sum(-1)
    comp = (A[:, :, None] + B[:, None, :]).reshape(len(x), I * I)
    W = rat["root_weights"]                        # [C, I*I], product order (i, j)
    ref = special.logsumexp(comp[:, None, :], b=W[None], axis=2)
    lp, am = oracle_eval(g, x)
    np.testing.assert_allclose(lp, ref, rtol=1e-12, atol=1e-10)
    assert np.array_equal(am, np.argmax(ref, axis=1))
