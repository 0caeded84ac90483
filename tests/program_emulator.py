"""Test-side reference interpreter of the node-program format (program.h).

It executes the records the preparer emits (``spn_build_program``) in fp64
numpy, vectorised over samples, so the preparer's code generation
(canonicalisation, partitioning, Sethi-Ullman stack allocation, slot
liveness, gather-LSE terms, chunked LSE) can be checked against the oracle on
the CPU, without a GPU.  It restates the record semantics documented in
program.h; it is not used by the product path.
"""
from __future__ import annotations

import numpy as np

NSP = 17
OPS = ["END", "LPUSH", "LACC", "ADD", "LSE1", "LSE2", "LSE3", "LSE4",
       "LDS", "LDG", "STS", "STG", "GLSE", "OUT", "NOP",
       "GPUSH1", "GPUSH2", "GPUSH3", "GPUSH4", "GACC1", "GACC2", "GACC3", "GACC4",
       "SLP2", "SLP3", "SLP4", "SLPU2", "SLPU3"]
SLOT_GLOBAL = 0x80000000
SLOT_NONE = 0xFFFFFFFF


def _f32(u):
    return float(np.array([u], dtype=np.uint32).view(np.float32)[0])


def _lse(vals):
    v = np.stack(vals)
    m = np.max(np.where(np.isnan(v), -np.inf, v), axis=0)
    m = np.maximum(m, -1e30)
    with np.errstate(invalid="ignore", over="ignore", divide="ignore"):
        s = np.sum(np.exp2(v - m), axis=0)
        return m + np.log2(s)


def emulate(prog: dict, x: np.ndarray, n_roots: int, marginal: bool, K: int,
            x_in_smem: bool):
    """Returns ln p [N, R] (float64)."""
    rec = prog["records"]
    toff = prog["task_off"]
    tables = prog["tables"].astype(np.float64)
    edges = prog["edges"]
    N = x.shape[0]
    xd = x.astype(np.float64)
    tpw = 32 * K + 4
    slot_bytes = 32 * K * 4
    stack = np.zeros((NSP, N))
    sslots: dict = {}
    gslots: dict = {}
    out = np.full((N, n_roots), np.nan)

    def feat(arg):
        return arg // (tpw * 4) if x_in_smem else arg // 4

    def slot_get(ref):
        if ref & SLOT_GLOBAL:
            return gslots[(ref & ~SLOT_GLOBAL) // slot_bytes]
        return sslots[ref // slot_bytes]

    for t in range(len(toff) - 1):
        pc = int(toff[t])
        while True:
            r = rec[pc]
            pc += 1
            xw = int(r["x"])
            case = xw & 511
            arg = xw >> 9
            op, sp = OPS[case // NSP] if case // NSP < len(OPS) else "BAD", case % NSP
            if op == "END":
                break
            if op.startswith("SLP"):
                if op.startswith("SLPU"):
                    k = int(op[4])
                    Cs = [_f32(r["z"]), _f32(r["w"])]
                    if k == 3:
                        Cs.append(_f32(rec[pc]["x"]))
                    pc += 1                   # feature-offset record (offsets repeat below)
                    arg = 2 | (2 << 3) | ((2 << 6) if k == 3 else 0)
                else:
                    k = int(op[3])
                    Cs = [_f32(r["z"]), _f32(r["w"])]
                    if k >= 3:
                        Cs += [_f32(rec[pc]["x"]), _f32(rec[pc]["y"])]
                        pc += 1
                vals = []
                for ci in range(k):
                    acc = np.full(N, Cs[ci])
                    for _ in range((arg >> (3 * ci)) & 7):
                        q = rec[pc]
                        pc += 1
                        xv = xd[:, feat(int(q["x"]))]
                        a, b, c = _f32(q["y"]), _f32(q["z"]), _f32(q["w"])
                        t = a * xv - b
                        acc = acc - (np.where(np.isnan(xv), c, t * t) if marginal else t * t)
                    vals.append(acc)
                stack[sp] = _lse(vals) + _f32(r["y"])
                continue
            if op[:5] in ("GPUSH", "GACC1", "GACC2", "GACC3", "GACC4"):
                ng, nd = int(op[-1]), 0
                op = "LPUSH" if op.startswith("GPUSH") else "LACC"
            elif op in ("LPUSH", "LACC"):
                ng, nd = arg, int(r["z"])
            if op in ("LPUSH", "LACC"):
                C = _f32(r["y"])
                acc = np.full(N, C)
                for i in range(ng):
                    q = rec[pc]
                    pc += 1
                    xv = xd[:, feat(int(q["x"]))]
                    a, b, c = _f32(q["y"]), _f32(q["z"]), _f32(q["w"])
                    t = a * xv - b
                    if marginal:
                        acc = acc - np.where(np.isnan(xv), c, t * t)
                    else:
                        acc = acc - t * t
                for i in range(nd):
                    q = rec[pc]
                    pc += 1
                    xv = xd[:, feat(int(q["x"]))]
                    off, lo, nk = int(q["y"]), int(np.int32(np.uint32(q["z"]))), int(q["w"])
                    ok = (xv >= lo) & (xv < lo + nk)
                    idx = np.where(ok, np.floor(np.where(ok, xv, lo)) - lo, 0).astype(np.int64)
                    v = np.where(ok, tables[off + idx], -np.inf)
                    v = np.where(np.isnan(xv), 0.0 if marginal else np.nan, v)
                    acc = acc + v
                if op == "LPUSH":
                    stack[sp] = acc
                else:
                    stack[sp - 1] = stack[sp - 1] + acc
            elif op == "ADD":
                stack[sp - 2] = stack[sp - 2] + stack[sp - 1] + _f32(r["y"])
            elif op.startswith("LSE"):
                n = int(op[3])
                bias = _f32(r["y"])
                if n == 1:
                    stack[sp - 1] = stack[sp - 1] + bias
                else:
                    stack[sp - n] = _lse([stack[sp - n + i] for i in range(n)]) + bias
            elif op == "LDS":
                stack[sp] = sslots[arg // slot_bytes] + _f32(r["y"])
            elif op == "LDG":  # global slot offsets ride in z (32 bits)
                stack[sp] = gslots[int(r["z"]) // slot_bytes] + _f32(r["y"])
            elif op == "STS":
                sslots[arg // slot_bytes] = stack[sp - 1].copy()
            elif op == "STG":
                gslots[int(r["z"]) // slot_bytes] = stack[sp - 1].copy()
            elif op == "GLSE":
                off = int(r["y"]) | (int(r["z"]) << 32)
                n = int(r["w"])
                vals = []
                for e in edges[off:off + n]:
                    v = slot_get(int(e["a"])).copy()
                    if int(e["b"]) != SLOT_NONE:
                        v = v + slot_get(int(e["b"]))
                    vals.append(v + float(e["lw"]))
                stack[sp] = _lse(vals)
            elif op == "OUT":
                out[:, arg] = stack[sp - 1] * np.log(2.0)
            elif op == "NOP":
                pass
            else:
                raise ValueError(f"bad record {pc - 1}: case {case}")
    return out
