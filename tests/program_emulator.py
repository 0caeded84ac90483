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
OPS = ["END", "GPUSH", "GACC", "DPUSH", "DACC", "ADD", "LSE1", "LSE2", "LSE3", "LSE4",
       "LDS", "LDG", "STS", "STG", "GLSE", "OUT", "NOP"]
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
            if op in ("GPUSH", "GACC"):
                xv = xd[:, feat(arg)]
                a, b, c = _f32(r["y"]), _f32(r["z"]), _f32(r["w"])
                v = c - (a * xv - b) ** 2
                if marginal:
                    v = np.where(np.isnan(xv), 0.0, v)
                if op == "GPUSH":
                    stack[sp] = v
                else:
                    stack[sp - 1] = stack[sp - 1] + v
            elif op in ("DPUSH", "DACC"):
                xv = xd[:, feat(arg)]
                off, lo, nk = int(r["y"]), int(np.int32(np.uint32(r["z"]))), int(r["w"])
                ok = (xv >= lo) & (xv < lo + nk)
                idx = np.where(ok, np.floor(np.where(ok, xv, lo)) - lo, 0).astype(np.int64)
                v = np.where(ok, tables[off + idx], -np.inf)
                v = np.where(np.isnan(xv), 0.0 if marginal else np.nan, v)
                if op == "DPUSH":
                    stack[sp] = v
                else:
                    stack[sp - 1] = stack[sp - 1] + v
            elif op == "ADD":
                stack[sp - 2] = stack[sp - 2] + stack[sp - 1]
            elif op.startswith("LSE"):
                n = int(op[3])
                w = [_f32(r["y"]), _f32(r["z"]), _f32(r["w"])]
                if n == 4:
                    w.append(_f32(rec[pc]["x"]))
                    pc += 1
                if n == 1:
                    stack[sp - 1] = stack[sp - 1] + w[0]
                else:
                    stack[sp - n] = _lse([stack[sp - n + i] + w[i] for i in range(n)])
            elif op == "LDS":
                stack[sp] = sslots[arg // slot_bytes]
            elif op == "LDG":
                stack[sp] = gslots[arg // slot_bytes]
            elif op == "STS":
                sslots[arg // slot_bytes] = stack[sp - 1].copy()
            elif op == "STG":
                gslots[arg // slot_bytes] = stack[sp - 1].copy()
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
