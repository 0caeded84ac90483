"""Launch-configuration sweep of the generic evaluator on one config
(kernel time by CUDA events, L2 flushed between reps)."""
import argparse
import json
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402
import paper_conf_cgo_sommera022_b200 as spnb  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="C2")
ap.add_argument("--marginal", action="store_true")
ap.add_argument("--combos", default="4:384,4:256,4:128,2:512,2:384,2:256,1:512")
ap.add_argument("--reps", type=int, default=10)
a = ap.parse_args()
g, x, n = bench.make_workload(a.config, 0, a.marginal)
G = spnb.Graph(g)
xd = torch.from_numpy(x).cuda()
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
for combo in a.combos.split(","):
    K, B = map(int, combo.split(":"))
    try:
        P = spnb.Plan(G, samples_per_thread=K, block_threads=B)
    except Exception as e:  # noqa: BLE001
        print(json.dumps({"K": K, "block": B, "error": str(e)}))
        continue
    out = torch.empty((n, g.n_roots), device="cuda")
    for _ in range(3):
        P.infer(xd, marginal=a.marginal, out=out, want_argmax=False)
    ts = []
    for _ in range(a.reps):
        flush.fill_(1)
        s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        s.record()
        P.infer(xd, marginal=a.marginal, out=out, want_argmax=False)
        e.record()
        torch.cuda.synchronize()
        ts.append(s.elapsed_time(e))
    ts.sort()
    info = P.info()
    ms = ts[len(ts) // 2]
    print(json.dumps({"K": K, "block": B, "grid": info["grid"], "smem": info["smem_bytes"],
                      "ms": ms, "samples_per_s": n / ms * 1e3,
                      "mufu_frac": info["mufu_per_sample"] * n / (ms / 1e3) / (16 * 148 * 1.965e9)}),
          flush=True)
