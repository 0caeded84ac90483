"""Summarise an `ncu --set full` capture (.ncu-rep) into profiles/ncu_<cfg>.json
(the file bench.py reads `roofline.traffic` from) and summarise an ncu launch
list (--metrics gpu__time_duration.sum --csv) into per-kernel shares.

usage: python scripts/ncu_summary.py full <rep> <config> <algorithmic_bytes> <capture note> > profiles/ncu_C2.json
       python scripts/ncu_summary.py launches <csv>  > profiles/rNN_ncu_launches_<cfg>_summary.json
"""
import csv
import io
import json
import subprocess
import sys

KEYS = [
    "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
    "sm__inst_executed_pipe_xu.avg.pct_of_peak_sustained_active",
    "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active",
    "sm__inst_executed_pipe_fma.avg.pct_of_peak_sustained_active",
    "sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active",
    "sm__pipe_tensor_op_hmma_cycles_active.avg.pct_of_peak_sustained_active",
    "sm__pipe_tc_cycles_active.avg.pct_of_peak_sustained_active",
    "sm__inst_issued.avg.pct_of_peak_sustained_active",
    "sm__warps_active.avg.pct_of_peak_sustained_active",
    "launch__registers_per_thread", "launch__grid_size", "launch__block_size",
    "smsp__inst_executed.sum", "thread_inst_executed",
    "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum",
    "lts__t_bytes.sum", "sm__cycles_elapsed.avg.per_second",
    "lts__t_sector_hit_rate.pct", "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum.pct_of_peak_sustained_elapsed",
    "TPC.TriageCompute.sm__pipe_tensor_cycles_active_realtime.avg.pct_of_peak_sustained_elapsed",
]
UNIT = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}


def full(rep, cfg, alg_bytes, note):
    raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True,
                         text=True, check=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    h, u, v = rows[0], rows[1], rows[2]
    m = {}
    for k in KEYS + [k for k in h if "average_warps_issue_stalled" in k and k.endswith("ratio")]:
        if k in h:
            i = h.index(k)
            m[k] = {"value": v[i], "unit": u[i]}
    dram = sum(float(m[k]["value"].replace(",", "")) * UNIT.get(m[k]["unit"], 1)
               for k in ("dram__bytes_read.sum", "dram__bytes_write.sum") if k in m)
    return {"kernel": v[h.index("Kernel Name")], "config": cfg, "capture": note,
            "dram_bytes_per_launch": dram, "algorithmic_bytes_per_launch": alg_bytes,
            "metrics": m}


def launches(path):
    text = open(path).read()
    text = text[text.index('"ID"'):]
    agg = {}
    for r in csv.DictReader(io.StringIO(text)):
        if r["Metric Name"] != "gpu__time_duration.sum":
            continue
        t = float(r["Metric Value"].replace(",", "")) * (1e-3 if r["Metric Unit"] == "ns" else 1)
        a = agg.setdefault(r["Kernel Name"][:80], [0, 0.0])
        a[0] += 1
        a[1] += t
    tot = sum(a[1] for a in agg.values())
    return {k: {"launches": a[0], "mean_us": a[1] / a[0], "share": a[1] / tot} for k, a in agg.items()}


if __name__ == "__main__":
    if sys.argv[1] == "full":
        out = full(sys.argv[2], sys.argv[3], float(sys.argv[4]), sys.argv[5])
    else:
        out = launches(sys.argv[2])
    json.dump(out, sys.stdout, indent=1)
    print()
