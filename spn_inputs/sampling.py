"""Seeded data generation: ancestral sampling from an SPN plus the
perturbations the configs call for (outliers, out-of-support values, NaN
masks for marginal queries).  No inference arithmetic here."""
from __future__ import annotations

import numpy as np

from .graph import FlatSPN, GAUSSIAN, CATEGORICAL, HISTOGRAM, SUM, PRODUCT


def ancestral_sample(g: FlatSPN, n: int, seed: int, root_probs=None):
    """Draw ``n`` samples top-down: pick a root (uniform unless given), at a
    sum pick one child with probability w_i / sum(w), at a product visit all
    children, at a leaf draw from its distribution.  Returns (x [n,F] float32,
    labels [n] int64).  Features never reached stay NaN (cannot happen for a
    complete SPN)."""
    rng = np.random.default_rng(seed)
    F = g.n_features
    x = np.full((n, F), np.nan, dtype=np.float64)
    R = g.n_roots
    if R > 1:
        p = np.full(R, 1.0 / R) if root_probs is None else np.asarray(root_probs, float)
        labels = rng.choice(R, size=n, p=p)
    else:
        labels = np.zeros(n, dtype=np.int64)
    stack = []
    for r in range(R - 1, -1, -1):
        idx = np.nonzero(labels == r)[0]
        if len(idx):
            stack.append((int(g.roots[r]), idx))
    kind = g.kind
    while stack:
        u, idx = stack.pop()
        k = int(kind[u])
        if k == PRODUCT:
            for c in g.child_list(u)[::-1]:
                stack.append((int(c), idx))
        elif k == SUM:
            ch = g.child_list(u)
            w = np.asarray(g.weight_list(u), dtype=np.float64)
            w = w / w.sum()
            pick = rng.choice(len(ch), size=len(idx), p=w)
            order = np.argsort(pick, kind="stable")
            counts = np.bincount(pick, minlength=len(ch))
            starts = np.concatenate([[0], np.cumsum(counts)])
            for j in range(len(ch) - 1, -1, -1):
                if counts[j]:
                    stack.append((int(ch[j]), idx[order[starts[j]:starts[j + 1]]]))
        else:
            f = int(g.feature[u])
            prm = g.param_list(u)
            if k == GAUSSIAN:
                x[idx, f] = rng.normal(prm[0], prm[1], size=len(idx))
            elif k == CATEGORICAL:
                pr = np.asarray(prm, float)
                x[idx, f] = rng.choice(len(pr), size=len(idx), p=pr / pr.sum())
            elif k == HISTOGRAM:
                bk = np.asarray(prm, float).reshape(-1, 3)
                mass = bk[:, 2] * (bk[:, 1] - bk[:, 0])
                j = rng.choice(len(bk), size=len(idx), p=mass / mass.sum())
                lo = bk[j, 0]
                width = (bk[j, 1] - bk[j, 0]).astype(np.int64)
                x[idx, f] = lo + np.floor(rng.random(len(idx)) * width)
            else:
                raise ValueError(f"bad kind {k}")
    return x.astype(np.float32), labels


def add_outliers(x: np.ndarray, frac: float, seed: int, lo=-10.0, hi=10.0):
    """Replace a fraction of entries by U[lo, hi] (config 2 recipe)."""
    rng = np.random.default_rng(seed)
    m = rng.random(x.shape) < frac
    y = x.copy()
    y[m] = rng.uniform(lo, hi, size=int(m.sum())).astype(np.float32)
    return y


def nan_mask(x: np.ndarray, p: float, seed: int):
    """i.i.d. missing features (NaN = missing, reading c6)."""
    rng = np.random.default_rng(seed)
    y = x.copy()
    y[rng.random(x.shape) < p] = np.nan
    return y


def toy_data(n: int, seed: int = 1001, oos_frac: float = 0.01):
    """Config 1: x0 ~ U{0,1}, x1 ~ U{0,1,2}, x2 ~ U{0..3}, with a fraction
    of out-of-support values (-1 or K) to reach log 0 = -inf."""
    rng = np.random.default_rng(seed)
    doms = [2, 3, 4]
    x = np.stack([rng.integers(0, K, size=n) for K in doms], axis=1).astype(np.float32)
    m = rng.random(x.shape) < oos_frac
    bad = np.where(rng.random(x.shape) < 0.5, -1.0, np.array(doms, float)[None, :])
    x[m] = bad[m]
    return x


def uniform_chunked(n: int, F: int, seed: int, start: int = 0, chunk: int = 65536):
    """Counter-based U[0,1] data, one generator per 65,536-sample chunk so any
    shard [start, start+n) is reproducible independently (config 5 recipe,
    SURVEY §8(d))."""
    out = np.empty((n, F), np.float32)
    pos = start
    while pos < start + n:
        c = pos // chunk
        c0 = c * chunk
        rng = np.random.default_rng([seed, c])
        block = rng.random((chunk, F), dtype=np.float32)
        a = pos - c0
        b = min(chunk, start + n - c0)
        out[pos - start:pos - start + (b - a)] = block[a:b]
        pos += b - a
    return out
