"""Small inference calls for compute-sanitizer runs (memcheck / racecheck /
synccheck), one kernel family per case:
  python scripts/sanitize_cases.py v2|v2tc|v1|interp|compiled|compiled_lin
(v2: FP32 FMA leaves, the default; v2tc: tensor-core leaves)"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_cgo_sommera022_b200 as spnb  # noqa: E402
from spn_inputs import ancestral_sample, nan_mask, rat_spn, speaker_spn, toy_spn, toy_data  # noqa: E402

case = sys.argv[1]
if case in ("v2", "v2tc", "v1"):
    g = rat_spn(11, F=64, D=3, R=2, S=8, I=16, C=5)
    opt = {"layered_path": 2, "layered_kernel": 1 if case == "v1" else 2, "leaf_tc": 2 if case == "v2tc" else 0}
    n = 300
elif case == "interp":
    g = rat_spn(7, F=64, D=3, R=3, S=6, I=8, C=4)
    opt = {"layered_path": 1, "compiled_path": 1, "max_task_nodes": 400}
    n = 700
elif case == "compiled":
    g, opt, n = speaker_spn(2001), {}, 5000
else:
    g, opt, n = toy_spn(), {"value_space": 2}, 5000
x = toy_data(n, seed=3) if case == "compiled_lin" else ancestral_sample(g, n, 1)[0]
P = spnb.Plan(spnb.Graph(g), **opt)
xd = torch.from_numpy(x).cuda()
for marg in (False, True):
    out, am = P.infer(xd if not marg else torch.from_numpy(nan_mask(x, 0.2, 2)).cuda(), marginal=marg)
torch.cuda.synchronize()
print(case, P.info()["path"], P.info()["layered_kernel"], P.info()["leaf_tc"], "ok", float(out.float().mean()))
