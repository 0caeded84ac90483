"""Test-side reference executor of the v2 layered plan (``spn_build_layered2``,
kernel rat2.cu), in fp64 numpy with the kernel's f16 operand rounding.  It
restates the step semantics (LEAF / BOT / UP, TMEM activation slots, per-sum
weight scale exponents, the 2^15 shift of the B-side exps) so the detector,
the weight images and the slot schedule can be checked against the oracle on
the CPU.  Not used by the product path."""
from __future__ import annotations

import numpy as np

EB_SHIFT = 15.0


def _img_index(row, k, rows):
    """f16-element index of (row, k) in a K-major no-swizzle operand image."""
    return (k // 8) * (rows * 8) + (row // 8) * 64 + (row % 8) * 8 + (k % 8)


def _f16_split(v, prec):
    hi = v.astype(np.float16).astype(np.float64)
    if prec == 3:
        lo = (v - hi).astype(np.float16).astype(np.float64)
        return hi + lo
    return hi


def _decode_weights(plan, st, prec):
    """W[s, i, j] from the group images: groups alternate between the A and
    B accumulator sizes (spg_a / spg_b sums, ncol_a / ncol_b columns), each
    stored as [hi, lo]."""
    na, nb, S = int(st["na"]), int(st["nb"]), int(st["n_out"])
    kpad = int(st["kpad"])
    wimg = plan["wimg"]
    W = np.zeros((S, na, nb))
    off = int(st["w_off"]) // 2
    for g in range(int(st["n_groups"])):
        b = g & 1
        ncol = int(st["ncol_b"] if b else st["ncol_a"])
        spg = int(st["spg_b"] if b else st["spg_a"])
        s_first = (g // 2) * int(st["spg_a"] + st["spg_b"]) + (int(st["spg_a"]) if b else 0)
        gel = ncol * kpad
        hi = wimg[off:off + gel].astype(np.float64)
        lo = wimg[off + gel:off + 2 * gel].astype(np.float64)
        off += 2 * gel
        wg = hi + (lo if prec == 3 else 0.0)
        for sl in range(spg):
            s = s_first + sl
            if s >= S:
                break
            for i in range(na):
                row = sl * na + i
                idx = [_img_index(row, j, ncol) for j in range(nb)]
                W[s, i, :] = wg[idx]
    return W


def _leaf_tc(plan, st, xd, marginal):
    """Tensor-core leaf variant: L[i, m] = sum_k F[m, k] P[k, i] with the
    features F = (x~^2, x~ per variable; 1 or the observed indicators) and
    the parameter image decoded from the plan, both split hi/lo in f16 and
    multiplied as F_h P_h + F_h P_l + F_l P_h (the kernel's three passes)."""
    I, lvp = plan["I"], plan["lvp"]
    V = int(st["n_vars"])
    N = xd.shape[0]
    NL = 48
    K = plan["kl_m"] if marginal else plan["kl_j"]
    fp = plan["fparams"].astype(np.float64)
    M = fp[int(st["blk_off"]):int(st["blk_off"]) + lvp]
    off = int(st["w_off"]) // 2 + (2 * int(st["wbytes_a"]) // 2 if marginal else 0)
    part = NL * K
    idx = np.array([[_img_index(n, k, NL) for n in range(NL)] for k in range(K)])
    Ph = plan["wimg"][off:off + part].astype(np.float64)[idx]
    Pl = plan["wimg"][off + part:off + 2 * part].astype(np.float64)[idx]
    F = np.zeros((N, K))
    for v in range(V):
        xv = xd[:, int(plan["vars"][int(st["vars_off"]) + v])]
        xt = (xv.astype(np.float32) - np.float32(M[v])).astype(np.float64)
        if marginal:
            obs = ~np.isnan(xt)
            xt = np.where(obs, xt, 0.0)
            F[:, 2 * lvp + v] = obs
        F[:, 2 * v] = xt * xt
        F[:, 2 * v + 1] = xt
    if not marginal:
        F[:, 2 * lvp] = 1.0
    Fh = F.astype(np.float16).astype(np.float64)
    Fl = (F - Fh).astype(np.float16).astype(np.float64)
    Fl[:, 2 * lvp:] = 0.0   # constant / indicator columns are exact
    L = Fh @ Ph + Fh @ Pl + Fl @ Ph
    return L[:, :I].T


def emulate_layered2(plan: dict, x: np.ndarray, marginal: bool = False, prec: int = 3):
    steps, vars_, fp = plan["steps"], plan["vars"], plan["fparams"].astype(np.float64)
    C, I = plan["C"], plan["I"]
    N = x.shape[0]
    xd = x.astype(np.float64)
    slots = {}
    racc = np.full((C, N), -np.inf)
    pending = []   # leaf outputs of the current bottom partition
    K0 = 0.5 * np.log2(np.log(2.0) / np.pi)
    with np.errstate(invalid="ignore", divide="ignore", over="ignore"):
        for st in steps:
            t = int(st["type"])
            if t == 0 and plan.get("leaf_tc"):
                pending.append(_leaf_tc(plan, st, xd, marginal))
                continue
            if t == 0:
                V = int(st["n_vars"])
                blk = fp[int(st["blk_off"]):int(st["blk_off"]) + int(st["blk_floats"])]
                ab = blk[:2 * V * I].reshape(V, I, 2)
                acc = np.tile(blk[2 * V * I:2 * V * I + I][:, None], (1, N))
                for v in range(V):
                    xv = xd[:, int(vars_[int(st["vars_off"]) + v])]
                    tt = ab[v, :, 0:1] * xv[None, :] - ab[v, :, 1:2]
                    if marginal:
                        cv = np.log2(ab[v, :, 0]) + K0
                        acc -= np.where(np.isnan(xv)[None, :], cv[:, None], tt * tt)
                    else:
                        acc -= tt * tt
                pending.append(acc)
                continue
            if t == 1:
                VA, VB = pending
                pending = []
            else:
                VA, VB = slots[int(st["slot_a"])], slots[int(st["slot_b"])]
            ha = np.max(VA, axis=0)
            hb = np.max(VB, axis=0) - EB_SHIFT
            ea = np.exp2(VA - np.maximum(ha, -1e30))
            eb = _f16_split(np.exp2(VB - np.maximum(hb + EB_SHIFT, -1e30) + EB_SHIFT), prec)
            W = _decode_weights(plan, st, prec)
            ks = fp[int(st["blk_off"]):int(st["blk_off"]) + int(st["n_out"])]
            T = np.einsum("jm,sij->sim", eb, W)
            val = (ha + hb)[None, :] + np.log2(np.einsum("im,sim->sm", ea, T)) - ks[:, None]
            if int(st["root"]):
                for s in range(int(st["n_out"])):
                    c = int(plan["root_map"][s])
                    racc[c] = np.logaddexp2(racc[c], val[s])
            else:
                slots[int(st["slot_out"])] = val
    return (racc * np.log(2.0)).T
