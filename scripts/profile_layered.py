"""Phase breakdown of the layered RAT-SPN kernel (SPNB_PROFILE=1 counters)."""
import os
import sys
import time

os.environ.setdefault("SPNB_PROFILE", "1")   # SPNB_PROFILE=0 for clean ncu captures
if os.environ["SPNB_PROFILE"] == "0":
    del os.environ["SPNB_PROFILE"]
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import bench  # noqa: E402
import paper_conf_cgo_sommera022_b200 as spnb  # noqa: E402
from spn_inputs import config_graph  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "C4"
prec = int(sys.argv[2]) if len(sys.argv) > 2 else 1
g = config_graph(cfg)
n = 18944 * 2
x = bench.device_uniform(n, g.n_features, 4002, 0, torch.device("cuda"))
P = spnb.Plan(spnb.Graph(g), tc_precision=prec)
print(P.info())
out, am = P.infer(x)
torch.cuda.synchronize()
t = time.perf_counter()
out, am = P.infer(x)
torch.cuda.synchronize()
print("ms", (time.perf_counter() - t) * 1e3, "samples/s", n / (time.perf_counter() - t))
P.close()  # prints the counters
