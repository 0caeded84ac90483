"""Where the host-buffer (e2e) path of the layered kernel loses time: C5 on
1M samples, device-resident vs host-buffer calls, certified vs raw single
pass, and the cost of a certification round with nothing flagged."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import bench  # noqa: E402
import paper_conf_cgo_sommera022_b200 as spnb  # noqa: E402
from spn_inputs import config_graph  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "C5"
n = int(sys.argv[2]) if len(sys.argv) > 2 else 1 << 20
g = config_graph(cfg)
G = spnb.Graph(g)
xd = bench.device_uniform(n, g.n_features, 5002, 0, torch.device("cuda"))
xh = xd.cpu().pin_memory()
for prec in (0, 1):
    P = spnb.Plan(G, tc_precision=prec)
    out, am = P.infer(xd)
    torch.cuda.synchronize()
    oh = torch.empty((n, P.n_roots), dtype=torch.float32).pin_memory()
    amh = torch.empty((n,), dtype=torch.int32).pin_memory()
    P.infer_host(xh, out=oh, argmax=amh)
    for what in ("device", "host"):
        ts = []
        for _ in range(3):
            torch.cuda.synchronize()
            t = time.perf_counter()
            if what == "device":
                P.infer(xd, out=out, argmax=am)
                torch.cuda.synchronize()
            else:
                P.infer_host(xh, out=oh, argmax=amh)
            ts.append(time.perf_counter() - t)
        print(cfg, "prec", prec, what, "ms", round(min(ts) * 1e3, 2), "samples/s", f"{n / min(ts):.3e}",
              "info", {k: P.info()[k] for k in ("chunk_samples", "certified")}, flush=True)
    P.close()
