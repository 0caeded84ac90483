"""fp64 CPU oracle for SPN inference -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py`` (cpu_baseline
and ``--impl reference`` legs) may import this package.  The product package
(paper_conf_cgo_sommera022_b200) never imports it and shares no code with it.

* ``oracle_eval``   -- the C recursive fp64 evaluator (spn_oracle.c), the
                       plain definition of PAPER.md §II-A (L34-L39) in log
                       space, OpenMP over samples.
* ``exact``         -- Fraction evaluator for discrete SPNs (exact rationals).

Every function is pinned by a `-m "not gpu"` test against something other
than itself (tests/test_oracle_pins.py); see DESIGN.md §Oracle.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "spn_oracle.c")
_LIB = os.path.join(_HERE, "_spn_oracle.so")
_lib = None


def build_oracle(force: bool = False) -> str:
    """Compile spn_oracle.c (gcc -O2 -fopenmp, no fast-math)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-fopenmp", "-fPIC", "-shared", "-std=c11",
                               "-D_GNU_SOURCE", _SRC, "-o", tmp, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


def _load():
    global _lib
    if _lib is None:
        build_oracle()
        lib = ctypes.CDLL(_LIB)
        P = ctypes.c_void_p
        I64 = ctypes.c_int64
        lib.oracle_eval.argtypes = [I64, P, P, P, P, P, P, P, P, P, I64, P,
                                    I64, P, I64, ctypes.c_int, P, P, ctypes.c_int]
        lib.oracle_eval.restype = ctypes.c_int
        lib.oracle_num_threads.restype = ctypes.c_int
        _lib = lib
    return _lib


def num_threads() -> int:
    return int(_load().oracle_num_threads())


def _ptr(a):
    return a.ctypes.data_as(ctypes.c_void_p)


def oracle_eval(g, x, marginal: bool = False, n_threads: int = 0, want_argmax=True):
    """Evaluate all roots of ``g`` (spn_inputs.FlatSPN) on samples ``x``
    ([N, >=F] float32).  Returns (logp [N, R] float64, argmax [N] int32)."""
    lib = _load()
    x = np.ascontiguousarray(x, dtype=np.float32)
    if x.ndim != 2:
        raise ValueError("x must be 2-D")
    N = x.shape[0]
    R = g.n_roots
    out = np.empty((N, R), dtype=np.float64)
    am = np.empty(N, dtype=np.int32) if want_argmax else None
    arrs = dict(
        kind=np.ascontiguousarray(g.kind, np.int32),
        feature=np.ascontiguousarray(g.feature, np.int32),
        child_begin=np.ascontiguousarray(g.child_begin, np.int64),
        n_children=np.ascontiguousarray(g.n_children, np.int32),
        param_begin=np.ascontiguousarray(g.param_begin, np.int64),
        n_params=np.ascontiguousarray(g.n_params, np.int32),
        children=np.ascontiguousarray(g.children, np.int64),
        weights=np.ascontiguousarray(g.weights, np.float64),
        params=np.ascontiguousarray(g.params, np.float64),
        roots=np.ascontiguousarray(g.roots, np.int64),
    )
    rc = lib.oracle_eval(g.n_nodes, _ptr(arrs["kind"]), _ptr(arrs["feature"]),
                         _ptr(arrs["child_begin"]), _ptr(arrs["n_children"]),
                         _ptr(arrs["param_begin"]), _ptr(arrs["n_params"]),
                         _ptr(arrs["children"]), _ptr(arrs["weights"]),
                         _ptr(arrs["params"]), R, _ptr(arrs["roots"]),
                         N, _ptr(x), x.shape[1], int(bool(marginal)), _ptr(out),
                         _ptr(am) if am is not None else None, int(n_threads))
    if rc != 0:
        raise MemoryError("oracle_eval allocation failed")
    return out, am
