"""Kernel / copy timeline of one host-buffer call (torch.profiler, CUPTI) on
C5: does the certified path keep the two-stream pipeline overlapped?"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
from torch.profiler import ProfilerActivity, profile  # noqa: E402

import bench  # noqa: E402
import paper_conf_cgo_sommera022_b200 as spnb  # noqa: E402
from spn_inputs import config_graph  # noqa: E402

out_dir = sys.argv[1]
n = 1 << 20
g = config_graph("C5")
G = spnb.Graph(g)
xd = bench.device_uniform(n, g.n_features, 5002, 0, torch.device("cuda"))
xh = xd.cpu().pin_memory()
for prec in (0, 1):
    P = spnb.Plan(G, tc_precision=prec)
    oh = torch.empty((n, P.n_roots), dtype=torch.float32).pin_memory()
    amh = torch.empty((n,), dtype=torch.int32).pin_memory()
    P.infer(xd)
    P.infer_host(xh, out=oh, argmax=amh)
    torch.cuda.synchronize()
    with profile(activities=[ProfilerActivity.CPU, ProfilerActivity.CUDA]) as prof:
        P.infer_host(xh, out=oh, argmax=amh)
        torch.cuda.synchronize()
    path = os.path.join(out_dir, f"e2e_trace_prec{prec}.json")
    prof.export_chrome_trace(path)
    ev = [e for e in json.load(open(path))["traceEvents"] if e.get("ph") == "X" and e.get("cat") in ("kernel", "gpu_memcpy", "gpu_memset")]
    t0 = min(e["ts"] for e in ev)
    rows = sorted((e["ts"] - t0, e["dur"], e.get("args", {}).get("stream"), e["name"][:40]) for e in ev)
    with open(os.path.join(out_dir, f"e2e_timeline_prec{prec}.txt"), "w") as f:
        for r in rows:
            f.write(f"{r[0]:10.0f} {r[1]:9.0f} s{r[2]} {r[3]}\n")
    print("prec", prec, "events", len(rows), "span us", max(r[0] + r[1] for r in rows))
    P.close()
