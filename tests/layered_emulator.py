"""Test-side reference executor of the layered (RAT-SPN) plan built by the
preparer (``spn_build_layered``), in fp64 numpy.  It restates the step
semantics of rat_eval.cu (LEAF / SUM / ROOT) so the detection, the weight
images and the buffer schedule can be checked against the oracle on the CPU.
Not used by the product path."""
from __future__ import annotations

import numpy as np

RT = 128


def _img_index(row, k, rows):
    """f16-element index of (row, k) in a K-major no-swizzle operand image."""
    return (k // 8) * (rows * 8) + (row // 8) * 64 + (row % 8) * 8 + (k % 8)


def emulate_layered(plan: dict, x: np.ndarray, n_roots: int, marginal: bool = False,
                    prec: int = 3):
    steps, vars_, fp = plan["steps"], plan["vars"], plan["fparams"].astype(np.float64)
    wimg = plan["wimg"]
    root_map = plan["root_map"]
    N = x.shape[0]
    xd = x.astype(np.float64)
    act = {}
    racc = np.full((n_roots, N), -np.inf)
    with np.errstate(invalid="ignore", divide="ignore", over="ignore"):
        for st in steps:
            t = int(st["type"])
            if t == 0:
                I, V = int(st["n_out"]), int(st["n_vars"])
                # pairs grouped as ab[v][g][k] = distribution g*DPT + k (8 groups,
                # DPT = I/8 padded to even)
                dpt = I // 8
                dptp = dpt + (dpt & 1)
                ab = fp[int(st["par_off"]):int(st["par_off"]) + V * 8 * dptp * 2].reshape(V, 8, dptp, 2)
                ab = ab[:, :, :dpt, :].reshape(V, I, 2)
                # per-(v, i) c = log2(a) + 0.5 log2(ln2/pi) (= -log2(sigma sqrt(2 pi)))
                cv = np.log2(ab[:, :, 0]) + 0.5 * np.log2(np.log(2.0) / np.pi)
                acc = np.tile(fp[int(st["cst_off"]):int(st["cst_off"]) + I][:, None], (1, N))
                for v in range(V):
                    xv = xd[:, int(vars_[int(st["vars_off"]) + v])]
                    tt = ab[v, :, 0:1] * xv[None, :] - ab[v, :, 1:2]
                    if marginal:
                        acc -= np.where(np.isnan(xv)[None, :], cv[v][:, None], tt * tt)
                    else:
                        acc -= tt * tt
                act[int(st["buf_out"])] = acc
                continue
            na, nb, S = int(st["na"]), int(st["nb"]), int(st["n_out"])
            VA, VB = act[int(st["buf_a"])], act[int(st["buf_b"])]
            ha = np.max(VA, axis=0)
            hb = np.max(VB, axis=0)
            ea = np.exp2(VA - np.maximum(ha, -1e30))
            eb = np.exp2(VB - np.maximum(hb, -1e30))
            # decode the weight images back to W[s, i, j]
            W = np.zeros((S, na, nb))
            ng, kpad, spg = int(st["n_group"]), int(st["k_pad"]), int(st["s_per_group"])
            gel = ng * kpad
            base = int(st["w_off"]) // 2
            rows = np.arange(ng)
            for g in range(int(st["n_groups"])):
                hi = wimg[base + 2 * g * gel: base + 2 * g * gel + gel].astype(np.float64)
                lo = wimg[base + 2 * g * gel + gel: base + 2 * (g + 1) * gel].astype(np.float64)
                wg = hi + (lo if prec == 3 else 0.0)
                for sl in range(spg):
                    s = g * spg + sl
                    if s >= S:
                        break
                    for i in range(na):
                        row = sl * na + i
                        idx = [_img_index(row, j, ng) for j in range(nb)]
                        W[s, i, :] = wg[idx]
            T = np.einsum("jm,sij->sim", eb, W)
            val = ha[None, :] + hb[None, :] + np.log2(np.einsum("im,sim->sm", ea, T))
            if t == 1:
                act[int(st["buf_out"])] = val
            else:
                for s in range(S):
                    c = int(root_map[s])
                    racc[c] = np.logaddexp2(racc[c], val[s])
    return (racc * np.log(2.0)).T
