"""Exact rational SPN oracle for discrete SPNs (TEST INFRASTRUCTURE ONLY).

Evaluates the SPN definition (§II-A) in linear
probability space with ``fractions.Fraction``: leaves give the exact
probability of the evidence (categorical: p_{floor x} for 0 <= x < K; histogram:
p of the half-open bucket containing x, readings c2/c3), products multiply,
sums take the weighted sum, marginalised (NaN) leaves give 1 (reading c6).
Only for discrete leaves with rational-representable parameters (the float
parameters are converted with ``Fraction(str(p))`` so 0.1 means 1/10).
"""
from __future__ import annotations

import math
from fractions import Fraction

CATEGORICAL = 1
HISTOGRAM = 2
SUM = 3
PRODUCT = 4


def _frac(v) -> Fraction:
    return Fraction(repr(float(v)))


def exact_probability(g, xs, marginal: bool = True):
    """xs: sequence of feature values (float, NaN = missing).  Returns a
    Fraction per root."""
    memo = {}

    def val(u):
        if u in memo:
            return memo[u]
        k = int(g.kind[u])
        if k == PRODUCT:
            v = Fraction(1)
            for c in g.child_list(u):
                v *= val(int(c))
        elif k == SUM:
            v = Fraction(0)
            for c, w in zip(g.child_list(u), g.weight_list(u)):
                v += _frac(w) * val(int(c))
        else:
            x = float(xs[int(g.feature[u])])
            p = g.param_list(u)
            if math.isnan(x):
                if not marginal:
                    raise ValueError("joint query with missing value")
                v = Fraction(1)
            elif k == CATEGORICAL:
                v = _frac(p[int(math.floor(x))]) if 0 <= x < len(p) else Fraction(0)
            elif k == HISTOGRAM:
                v = Fraction(0)
                for b in range(0, len(p), 3):
                    if p[b] <= x < p[b + 1]:
                        v = _frac(p[b + 2])
                        break
            else:
                raise ValueError("exact oracle supports discrete leaves only")
        memo[u] = v
        return v

    return [val(int(r)) for r in g.roots]


def exact_log(fr: Fraction) -> float:
    """ln of a non-negative Fraction (ln 0 = -inf), accurate for tiny values."""
    if fr == 0:
        return float("-inf")
    return math.log(fr.numerator) - math.log(fr.denominator)
