"""Timeline of CTA 0 of the layered v2 kernel (R2_TRACE variant build +
SPNB_PROFILE=1): every role's phase marks as (clock, warp, phase), saved
to an .npy for scripts/trace_report.py.
usage: SPNB_LIB=variants/libspnb_trace.so SPNB_PROFILE=1 python scripts/trace_layered.py C5 out.npy"""
import ctypes
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import bench  # noqa: E402
import paper_conf_cgo_sommera022_b200 as spnb  # noqa: E402
from spn_inputs import config_graph  # noqa: E402

cfg, out_path = sys.argv[1], sys.argv[2]
g = config_graph(cfg)
n = 148 * 128 * 2
x = bench.device_uniform(n, g.n_features, 4002, 0, torch.device("cuda"))
P = spnb.Plan(spnb.Graph(g), tc_precision=1)
lib = spnb.load_library()
buf = (ctypes.c_ulonglong * (2 * (1 << 17)))()
P.infer(x)
torch.cuda.synchronize()
lib.spnb_r2_trace(buf, 1 << 17)  # drop the first launch's events
P.infer(x)
torch.cuda.synchronize()
k = lib.spnb_r2_trace(buf, 1 << 17)
a = np.frombuffer(buf, dtype=np.uint64, count=2 * k).reshape(k, 2).copy()
a = a[a[:, 0] != 0]
np.save(out_path, a)
print("events", k)
P.close()
