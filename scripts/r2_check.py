"""GPU check of the v2 layered kernel (rat2.cu): parity against the fp64
oracle on small RAT-SPNs and a C4 sample, then timings of v1 / v2 on C4 / C5.
usage: python scripts/r2_check.py [parity|time|time1|ltc|ltctime|all]"""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import bench  # noqa: E402
import paper_conf_cgo_sommera022_b200 as spnb  # noqa: E402
from oracle import oracle_eval  # noqa: E402
from spn_inputs import ancestral_sample, config_graph, nan_mask, rat_spn  # noqa: E402

what = sys.argv[1] if len(sys.argv) > 1 else "all"


def err(a, ref):
    both_inf = np.isneginf(a) & np.isneginf(ref)
    e = np.abs(a - ref) / np.maximum(1.0, np.abs(ref))
    e[both_inf] = 0
    return float(np.nanmax(e))


if what in ("parity", "all"):
    for shape in [(32, 2, 2, 4, 8, 3), (64, 3, 3, 8, 16, 5), (24, 1, 1, 4, 8, 2), (96, 4, 2, 20, 40, 10)]:
        F, D, R, S, I, C = shape
        g = rat_spn(7, F=F, D=D, R=R, S=S, I=I, C=C)
        x, _ = ancestral_sample(g, 1000, 3)
        ref, _ = oracle_eval(g, x)
        refm, _ = oracle_eval(g, nan_mask(x, 0.2, 4), marginal=True)
        for prec in (0, 1):
            P = spnb.Plan(spnb.Graph(g), layered_path=2, tc_precision=prec, layered_kernel=2)
            xd = torch.from_numpy(x).cuda()
            out, am = P.infer(xd)
            outm, _ = P.infer(torch.from_numpy(nan_mask(x, 0.2, 4)).cuda(), marginal=True)
            torch.cuda.synchronize()
            print("shape", shape, "prec", prec, "info", P.info()["layered_kernel"],
                  "cert", P.info()["certified"], round(P.info()["cert_err"], 5),
                  "err", err(out.cpu().numpy(), ref), "marg err", err(outm.cpu().numpy(), refm),
                  flush=True)
    g = config_graph("C4")
    x, _ = ancestral_sample(g, 300, 4002)
    ref, _ = oracle_eval(g, x)
    for prec in (0, 1):
        P = spnb.Plan(spnb.Graph(g), tc_precision=prec, layered_kernel=2)
        out, am = P.infer(torch.from_numpy(x).cuda())
        torch.cuda.synchronize()
        print("C4 prec", prec, "err", err(out.cpu().numpy(), ref), "argmax agree",
              float((am.cpu().numpy() == ref.argmax(1)).mean()), flush=True)

if what == "time1":   # v2 single pass only (A/B of kernel variants)
    for cfg, n in (("C4", 100_000), ("C5", 18944 * 16)):
        g = config_graph(cfg)
        xd = bench.device_uniform(n, g.n_features, 4002, 0, torch.device("cuda"))
        P = spnb.Plan(spnb.Graph(g), tc_precision=1, layered_kernel=2)
        out, am = P.infer(xd)
        torch.cuda.synchronize()
        ts = []
        for _ in range(3):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            P.infer(xd, out=out, argmax=am)
            e1.record()
            torch.cuda.synchronize()
            ts.append(e0.elapsed_time(e1))
        print(cfg, "v2 prec 1 ms", round(min(ts), 3), "samples/s", f"{n / min(ts) * 1e3:.3e}",
              "mean logp", float(out.float().mean()), flush=True)

if what in ("time", "all"):
    for cfg, n in (("C4", 100_000), ("C5", 18944 * 16)):
        g = config_graph(cfg)
        G = spnb.Graph(g)
        xd = bench.device_uniform(n, g.n_features, 4002, 0, torch.device("cuda"))
        for kern, prec in ((2, 0), (2, 1), (1, 2)):
            P = spnb.Plan(G, tc_precision=prec, layered_kernel=kern)
            out, am = P.infer(xd)
            torch.cuda.synchronize()
            ts = []
            for _ in range(3):
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record()
                P.infer(xd, out=out, argmax=am)
                e1.record()
                torch.cuda.synchronize()
                ts.append(e0.elapsed_time(e1))
            ms = min(ts)
            print(cfg, "kernel", kern, "prec", prec, "ms", round(ms, 3), "samples/s", f"{n / ms * 1e3:.3e}",
                  "smem", P.info()["smem_bytes"], flush=True)
            if kern == 2 and prec == 1:
                o1 = out.clone()
            if kern == 1:
                print("   v1 vs v2(prec1) max abs diff", float((out - o1).abs().max()), flush=True)
            P.close()

if what == "ltc":   # tensor-core leaves (leaf_tc): parity small shapes + C4 sample, joint / marginal
    shapes = [(32, 2, 2, 4, 8, 3), (64, 3, 3, 8, 16, 5), (24, 1, 1, 4, 8, 2), (96, 4, 2, 20, 40, 10)]
    for shape in shapes:
        F, D, R, S, I, C = shape
        g = rat_spn(7, F=F, D=D, R=R, S=S, I=I, C=C)
        x, _ = ancestral_sample(g, 1000, 3)
        xm = nan_mask(x, 0.2, 4)
        ref, _ = oracle_eval(g, x)
        refm, _ = oracle_eval(g, xm, marginal=True)
        for ltc in (2, 1):
            P = spnb.Plan(spnb.Graph(g), layered_path=2, layered_kernel=2, leaf_tc=ltc)
            out, am = P.infer(torch.from_numpy(x).cuda())
            outm, _ = P.infer(torch.from_numpy(xm).cuda(), marginal=True)
            torch.cuda.synchronize()
            print("shape", shape, "leaf_tc", P.info()["leaf_tc"], "err", err(out.cpu().numpy(), ref),
                  "marg err", err(outm.cpu().numpy(), refm), flush=True)
    g = config_graph("C4")
    x, _ = ancestral_sample(g, 300, 4002)
    ref, _ = oracle_eval(g, x)
    for ltc in (2, 1):
        P = spnb.Plan(spnb.Graph(g), leaf_tc=ltc)
        out, am = P.infer(torch.from_numpy(x).cuda())
        torch.cuda.synchronize()
        o = out.cpu().numpy()
        print("C4 leaf_tc", P.info()["leaf_tc"], "err", err(o, ref), "max abs", float(np.abs(o - ref).max()),
              "argmax agree", float((am.cpu().numpy() == ref.argmax(1)).mean()), flush=True)

if what == "ltctime":   # certified v2, tensor-core leaves vs FMA leaves
    for cfg, n in (("C4", 100_000), ("C5", 18944 * 16)):
        g = config_graph(cfg)
        G = spnb.Graph(g)
        xd = bench.device_uniform(n, g.n_features, 4002, 0, torch.device("cuda"))
        outs = {}
        for ltc in (2, 1):
            P = spnb.Plan(G, leaf_tc=ltc)
            out, am = P.infer(xd)
            torch.cuda.synchronize()
            ts = []
            for _ in range(3):
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record()
                P.infer(xd, out=out, argmax=am)
                e1.record()
                torch.cuda.synchronize()
                ts.append(e0.elapsed_time(e1))
            outs[ltc] = out.clone()
            print(cfg, "leaf_tc", P.info()["leaf_tc"], "ms", round(min(ts), 3), "samples/s",
                  f"{n / min(ts) * 1e3:.3e}", "smem", P.info()["smem_bytes"], flush=True)
            P.close()
        d = (outs[2] - outs[1]).abs()
        print(cfg, "tc vs fma leaves: max abs diff", float(d.max()), "rel",
              float((d / outs[1].abs().clamp(min=1)).max()), flush=True)
