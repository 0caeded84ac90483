"""Print a window of the layered v2 CTA-0 timeline (scripts/trace_layered.py output).
usage: python scripts/trace_report.py trace.npy [start_event_fraction] [cycles] [warps]"""
import sys

import numpy as np

a = np.load(sys.argv[1])
frac = float(sys.argv[2]) if len(sys.argv) > 2 else 0.5
span = int(sys.argv[3]) if len(sys.argv) > 3 else 30000
warps = [int(v) for v in sys.argv[4].split(",")] if len(sys.argv) > 4 else [0, 4, 8, 12, 13, 14]
t = a[:, 0].astype(np.int64)
w = (a[:, 1] >> 8).astype(int)
k = (a[:, 1] & 255).astype(int)
o = np.argsort(t, kind="stable")
t, w, k = t[o] - t[o][0], w[o], k[o]
NAMES = {"leaf": {0: "in-wait", 1: "compute", 2: "shift", 3: "out-wait", 4: "exp+write"},
         "epi": {5: "step-setup", 0: "leaf-wait", 1: "up-phase1", 3: "sums", 2: "T_FULL-wait", 4: "tile-io", 6: "tmem-ld", 7: "dots+fin"},
         12: {7: "issue", 0: "in-slot-wait"}, 13: {0: "A-wait", 3: "issue", 1: "W-wait", 2: "T_EMPTY-wait", 4: "mma-issue", 5: "commit-T", 6: "commit-W"},
         14: {7: "issue", 2: "W-slot-wait"}}


def nm(wi, ki):
    d = NAMES["leaf"] if wi < 4 else NAMES["epi"] if wi < 12 else NAMES.get(wi, {})
    return d.get(ki, str(ki))


lo = t[int(len(t) * frac)]
last = {}
for ti, wi, ki in zip(t, w, k):
    if wi in warps and lo <= ti < lo + span:
        d = ti - last.get(wi, ti)
        print(f"{ti - lo:8d}  w{wi:<2d} {'':{4 * warps.index(wi)}}{nm(wi, ki):>13s} ({d})")
    last[wi] = ti
