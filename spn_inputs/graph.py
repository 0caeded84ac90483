"""Flat SPN graph container and an SPFlow-like builder.

This is the *input format* shared by the oracle and the CUDA path (each side
marshals these arrays itself; neither imports the other).  It holds no
inference arithmetic -- only structure and parameters.

Node kinds follow the HiSPN leaf/inner operations of PAPER.md Table I
(L88-169): gaussian (mean, stddev), categorical (probabilities), histogram
(buckets), weighted sum (weights), product.  Multiple roots are allowed
(SURVEY.md §8(c) reading c10).

Parameter layout per node (``params[param_begin : param_begin + n_params]``):
  GAUSSIAN     [mean, stddev]
  CATEGORICAL  [p_0, ..., p_{K-1}]
  HISTOGRAM    [lb_0, ub_0, p_0, lb_1, ub_1, p_1, ...]  half-open [lb, ub),
               integer bounds, p = probability of each integer value
               (reading c2)
Sum weights are ``weights[child_begin : child_begin + n_children]`` (linear,
not renormalised, reading c9).  ``weights`` entries of product edges are 0
and ignored.
"""
from __future__ import annotations

from dataclasses import dataclass, field
from typing import Sequence

import numpy as np

GAUSSIAN = 0
CATEGORICAL = 1
HISTOGRAM = 2
SUM = 3
PRODUCT = 4

KIND_NAMES = {GAUSSIAN: "gaussian", CATEGORICAL: "categorical",
              HISTOGRAM: "histogram", SUM: "sum", PRODUCT: "product"}


@dataclass
class FlatSPN:
    kind: np.ndarray          # int32 [n]
    feature: np.ndarray       # int32 [n]   (-1 for inner nodes)
    child_begin: np.ndarray   # int64 [n]
    n_children: np.ndarray    # int32 [n]
    param_begin: np.ndarray   # int64 [n]
    n_params: np.ndarray      # int32 [n]
    children: np.ndarray      # int64 [E]
    weights: np.ndarray       # float64 [E]
    params: np.ndarray        # float64 [P]
    roots: np.ndarray         # int64 [R]
    n_features: int
    meta: dict = field(default_factory=dict)

    @property
    def n_nodes(self) -> int:
        return int(self.kind.shape[0])

    @property
    def n_edges(self) -> int:
        return int(self.children.shape[0])

    @property
    def n_roots(self) -> int:
        return int(self.roots.shape[0])

    def child_list(self, u: int) -> np.ndarray:
        b = int(self.child_begin[u])
        return self.children[b:b + int(self.n_children[u])]

    def weight_list(self, u: int) -> np.ndarray:
        b = int(self.child_begin[u])
        return self.weights[b:b + int(self.n_children[u])]

    def param_list(self, u: int) -> np.ndarray:
        b = int(self.param_begin[u])
        return self.params[b:b + int(self.n_params[u])]

    def counts(self) -> dict:
        k = self.kind
        sums = k == SUM
        return {
            "nodes": self.n_nodes,
            "gaussian": int((k == GAUSSIAN).sum()),
            "categorical": int((k == CATEGORICAL).sum()),
            "histogram": int((k == HISTOGRAM).sum()),
            "sum": int(sums.sum()),
            "product": int((k == PRODUCT).sum()),
            "sum_edges": int(self.n_children[sums].sum()),
            "edges": self.n_edges,
            "roots": self.n_roots,
        }

    def mufu_per_sample(self) -> int:
        """Algorithmic MUFU count per sample: the max-shifted n-ary log-sum-exp
        of a sum with n > 1 children needs n - 1 ex2 (the shift term is exactly
        1) and 1 lg2 (SURVEY.md §8(a) row a4 counted n + 1)."""
        nc = self.n_children[self.kind == SUM].astype(np.int64)
        return int(nc[nc > 1].sum())

    def validate_basic(self) -> None:
        n = self.n_nodes
        for name in ("feature", "child_begin", "n_children", "param_begin", "n_params"):
            assert getattr(self, name).shape == (n,), name
        assert self.weights.shape == self.children.shape


class GraphBuilder:
    """Append-only builder (SPFlow-like DSL).  Returns node ids."""

    def __init__(self, n_features: int):
        self.n_features = int(n_features)
        self._kind: list[int] = []
        self._feature: list[int] = []
        self._cb: list[int] = []
        self._nc: list[int] = []
        self._pb: list[int] = []
        self._np: list[int] = []
        self._children: list[int] = []
        self._weights: list[float] = []
        self._params: list[float] = []

    def _node(self, kind, feature, children=(), weights=None, params=()):
        nid = len(self._kind)
        self._kind.append(kind)
        self._feature.append(feature)
        self._cb.append(len(self._children))
        self._nc.append(len(children))
        self._children.extend(int(c) for c in children)
        if weights is None:
            self._weights.extend([0.0] * len(children))
        else:
            assert len(weights) == len(children)
            self._weights.extend(float(w) for w in weights)
        self._pb.append(len(self._params))
        self._np.append(len(params))
        self._params.extend(float(p) for p in params)
        return nid

    def gaussian(self, feature: int, mean: float, stddev: float) -> int:
        return self._node(GAUSSIAN, feature, params=(mean, stddev))

    def categorical(self, feature: int, probs: Sequence[float]) -> int:
        return self._node(CATEGORICAL, feature, params=tuple(probs))

    def histogram(self, feature: int, buckets: Sequence[tuple]) -> int:
        flat = []
        for lb, ub, p in buckets:
            flat.extend((lb, ub, p))
        return self._node(HISTOGRAM, feature, params=flat)

    def sum(self, children: Sequence[int], weights: Sequence[float]) -> int:
        return self._node(SUM, -1, children=children, weights=weights)

    def product(self, children: Sequence[int]) -> int:
        return self._node(PRODUCT, -1, children=children)

    def build(self, roots: Sequence[int], meta: dict | None = None) -> FlatSPN:
        return FlatSPN(
            kind=np.asarray(self._kind, dtype=np.int32),
            feature=np.asarray(self._feature, dtype=np.int32),
            child_begin=np.asarray(self._cb, dtype=np.int64),
            n_children=np.asarray(self._nc, dtype=np.int32),
            param_begin=np.asarray(self._pb, dtype=np.int64),
            n_params=np.asarray(self._np, dtype=np.int32),
            children=np.asarray(self._children, dtype=np.int64),
            weights=np.asarray(self._weights, dtype=np.float64),
            params=np.asarray(self._params, dtype=np.float64),
            roots=np.asarray(list(roots), dtype=np.int64),
            n_features=self.n_features,
            meta=dict(meta or {}),
        )


def disjoint_union(graphs: Sequence[FlatSPN]) -> FlatSPN:
    """Put several SPNs over the same features into one multi-root graph
    (one root per input graph, in order).  Used for config 3's per-speaker
    SPN set (one SPN per speaker, compare likelihoods)."""
    F = graphs[0].n_features
    kinds, feats, cbs, ncs, pbs, nps, chs, ws, ps, roots = ([] for _ in range(10))
    node_off = 0
    edge_off = 0
    par_off = 0
    for g in graphs:
        assert g.n_features == F
        kinds.append(g.kind)
        feats.append(g.feature)
        cbs.append(g.child_begin + edge_off)
        ncs.append(g.n_children)
        pbs.append(g.param_begin + par_off)
        nps.append(g.n_params)
        chs.append(g.children + node_off)
        ws.append(g.weights)
        ps.append(g.params)
        roots.append(g.roots + node_off)
        node_off += g.n_nodes
        edge_off += g.n_edges
        par_off += g.params.shape[0]
    return FlatSPN(
        kind=np.concatenate(kinds).astype(np.int32),
        feature=np.concatenate(feats).astype(np.int32),
        child_begin=np.concatenate(cbs).astype(np.int64),
        n_children=np.concatenate(ncs).astype(np.int32),
        param_begin=np.concatenate(pbs).astype(np.int64),
        n_params=np.concatenate(nps).astype(np.int32),
        children=np.concatenate(chs).astype(np.int64),
        weights=np.concatenate(ws).astype(np.float64),
        params=np.concatenate(ps).astype(np.float64),
        roots=np.concatenate(roots).astype(np.int64),
        n_features=F,
        meta={"union_of": len(graphs)},
    )
