#!/usr/bin/env python
"""Benchmark: SPN inference samples/s on B200 (BASELINE.json metric).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config C2]
                    [--marginal] [--impl ours|reference]

A step is one pass of the whole hot path (spn_infer_* over one batch of the
config's samples, inputs resident in HBM).  Default workload: config C5 (a
RAT-SPN of 3,242,010 nodes over 784 features, 10 class roots, 10M samples,
joint + argmax) -- the largest configuration of BASELINE.json, the one the
north star's >= 7x-at-8-GPUs target is stated on; it fits one B200.  C5
scales strongly: the 10M samples are split over the N ranks and, at N > 1,
every step ends with the NCCL all-gather of the per-sample log-likelihoods
and argmax (the only collective), inside the timed region.
The other configs scale weakly (a full batch per rank).  The input (31 GB at
N = 1) is larger than L2; L2 is also flushed (256 MiB write) between timed
steps.  Prints ONE JSON line on rank 0.  ``--impl reference`` times the fp64
CPU oracle (the reference arm of this tier) on bounded samples of the same
workload.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "SPN inference samples/sec (joint & marginal) at 1/2/4/8 B200; % of HBM/MUFU roofline"
UNIT = "samples/s"


_N_OVERRIDE = {}


def CONFIGS_N(cfg: str) -> int:
    """Samples of a config (BASELINE.json sizes; --samples overrides, e.g. C1
    at 1e8 where the toy SPN becomes HBM-bound)."""
    from spn_inputs import CONFIGS
    return _N_OVERRIDE.get(cfg, CONFIGS[cfg]["n_samples"])


def _peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        return d, "measured"
    return {"hbm_gbs": 6650.0, "sm_max_mhz": 1965.0}, "fallback"


def samples_per_rank(cfg: str, world: int) -> tuple[int, str]:
    """C5 is a strong-scaling config (10M samples split over the GPUs,
    BASELINE.json configs[4]); the others are weak (a full batch per GPU)."""
    from spn_inputs import CONFIGS
    from paper_conf_cgo_sommera022_b200.parallel import shard_sizes
    n = CONFIGS_N(cfg)
    if cfg == "C5":
        return max(shard_sizes(n, world)), "strong"
    return n, "weak"


def device_uniform(n: int, F: int, seed: int, start: int, dev, chunk: int = 65536):
    """Counter-based U[0,1) features generated on the GPU, one generator per
    65,536-sample chunk (shard independent; the RAT-SPN throughput recipe)."""
    import torch
    x = torch.empty((n, F), dtype=torch.float32, device=dev)
    pos = start
    while pos < start + n:
        c = pos // chunk
        gen = torch.Generator(device=dev)
        gen.manual_seed(seed * 1_000_003 + c)
        blk = torch.rand((chunk, F), generator=gen, device=dev, dtype=torch.float32)
        a = pos - c * chunk
        b = min(chunk, start + n - c * chunk)
        x[pos - start:pos - start + (b - a)] = blk[a:b]
        pos += b - a
    return x


def make_workload(cfg: str, rank: int, marginal: bool, n_max: int | None = None):
    """Seeded graph + this rank's input batch (host numpy); RAT-SPN inputs
    are generated for the first n_max samples only when n_max is given."""
    from spn_inputs import (CONFIGS, config_graph, ancestral_sample, add_outliers, nan_mask,
                            toy_data, uniform_chunked)
    c = CONFIGS[cfg]
    g = config_graph(cfg)
    n = CONFIGS_N(cfg)
    if cfg == "C1":
        x = toy_data(n, seed=1001 + rank)
        if marginal:
            x = nan_mask(x, 0.2, 1002 + rank)
    elif cfg == "C2":
        x, _ = ancestral_sample(g, n, c["data_seed"] + 1000 * rank)
        x = add_outliers(x, 0.01, c["data_seed"] + 1 + 1000 * rank)
        if marginal:
            x = nan_mask(x, 0.2, c["data_seed"] + 2 + 1000 * rank)
    elif cfg == "C3":
        x, _ = ancestral_sample(g, n, c["data_seed"] + 1000 * rank)
        x = nan_mask(x, c["nan_p"], c["nan_seed"] + 1000 * rank)
    else:
        # RAT-SPN configs: counter-based U[0,1] features (the layered path's
        # work is data independent; parity tests use ancestral samples)
        x = uniform_chunked(min(n, n_max or n), g.n_features, c["data_seed"], start=rank * n)
    return g, x, n


class ClockSampler:
    """nvidia-smi sampling of SM clocks / throttle reasons during a region."""
    FIELDS = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown,"
              "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
              "clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int):
        self.index = index
        self.proc = None
        self.path = os.path.join("/tmp", f"spnb_clocks_{os.getpid()}.csv")

    def start(self):
        try:
            self.f = open(self.path, "w")
            self.proc = subprocess.Popen(
                ["nvidia-smi", f"--id={self.index}", f"--query-gpu={self.FIELDS}",
                 "--format=csv,noheader,nounits", "-lms", "50"], stdout=self.f,
                stderr=subprocess.DEVNULL)
        except Exception:
            self.proc = None

    def stop(self):
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        time.sleep(0.12)
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except Exception:
            self.proc.kill()
        self.f.close()
        sm, mx, reasons = [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for line in open(self.path):
            parts = [p.strip() for p in line.split(",")]
            if len(parts) < 7:
                continue
            try:
                sm.append(float(parts[0]))
                mx.append(float(parts[1]))
            except ValueError:
                continue
            for nm, v in zip(names, parts[3:7]):
                if v.lower().startswith("active"):
                    reasons.add(nm)
        os.unlink(self.path)
        return {"sm_mhz": statistics.median(sm) if sm else None,
                "sm_max_mhz": max(mx) if mx else None, "reasons": sorted(reasons),
                "samples": len(sm)}


def cpu_baseline(g, x, marginal, target_s=12.0):
    """The oracle as it stands, timed on this host's cores on a bounded
    sample (~target_s seconds)."""
    from oracle import oracle_eval, num_threads
    n0 = min(len(x), 16)
    while True:
        t = time.perf_counter()
        oracle_eval(g, x[:n0], marginal=marginal)
        dt = time.perf_counter() - t
        if dt > 0.5 or n0 >= len(x):
            break
        n0 = min(len(x), n0 * 8)
    n = int(min(len(x), max(n0, n0 * target_s / max(dt, 1e-6))))
    t = time.perf_counter()
    oracle_eval(g, x[:n], marginal=marginal)
    dt = time.perf_counter() - t
    return {"value": n / dt, "unit": UNIT, "cores": num_threads(), "kind": "oracle",
            "sample": f"first {n} of the {len(x)} samples of this workload, "
                      f"fp64 recursive oracle, {dt:.1f} s"}


def run_reference(args):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    from oracle import oracle_eval, num_threads, build_oracle
    build_oracle()
    g, x, n = make_workload(args.config, 0, args.marginal,
                            n_max=4096 if args.config in ("C4", "C5") else None)
    # per step: a bounded sample sized so the whole run takes a few minutes
    # (calibrated from a growing probe: one C5 sample costs ~1 s of one core)
    n0 = min(n, 16)
    while True:
        t = time.perf_counter()
        oracle_eval(g, x[:n0], marginal=args.marginal)
        dt = time.perf_counter() - t
        if dt > 1.0 or n0 >= min(n, 4096):
            break
        n0 = min(n, n0 * 4)
    per = dt / n0
    budget = 150.0 / max(1, args.steps + args.warmup)
    m = int(max(16, min(x.shape[0], budget / max(per, 1e-9))))
    for i in range(args.warmup):
        oracle_eval(g, x[:m], marginal=args.marginal)
    ts = []
    for i in range(args.steps):
        off = (i * m) % max(1, x.shape[0] - m + 1)
        t = time.perf_counter()
        oracle_eval(g, x[off:off + m], marginal=args.marginal)
        ts.append(time.perf_counter() - t)
    tot = sum(ts)
    val = m * args.steps / tot
    line = {"impl": "reference", "metric": METRIC, "value": val, "unit": UNIT,
            "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": 1e3 * tot / args.steps, "higher_is_better": True,
            "scaling": "strong" if args.config == "C5" else "weak", "vs_baseline": None,
            "dtype": "f64", "data": "synthetic",
            "config": _config_dict(args, g, n, args.gpus,
                                   "strong" if args.config == "C5" else "weak"),
            "cpu_baseline": {"value": val, "unit": UNIT, "cores": num_threads(),
                             "kind": "oracle",
                             "sample": f"{m} samples per step of the {args.config} workload"},
            "e2e": {"value": val, "unit": UNIT, "h2d_bytes_per_step": 0,
                    "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def _config_dict(args, g, n, world=1, scaling="weak"):
    from spn_inputs import CONFIGS
    c = g.counts()
    desc = CONFIGS[args.config]["desc"]
    if args.config in _N_OVERRIDE:
        desc += f" [--samples {_N_OVERRIDE[args.config]}]"
    query = "marginal" if args.marginal else "joint"
    d = {"workload": f"{args.config}: {desc}, {query}",
         "query": "marginal" if args.marginal else "joint",
         "samples_per_gpu": n, "n_features": g.n_features, "n_roots": g.n_roots,
         "graph_nodes": c["nodes"], "sum_edges": c["sum_edges"],
         "l2": "flushed between timed steps (256 MiB write)",
         "parallelism": f"dp{world} (sample sharding)"}
    if scaling == "strong":
        d["samples_total"] = CONFIGS_N(args.config)
        d["l2"] = ("inputs larger than L2 (31 GB / N) and L2 flushed between timed steps "
                   "(256 MiB write)")
    return d


def launches_per_step(info: dict, n: int, want_am: bool) -> int:
    """Kernels of this library launched by one inference call (see api.cpp)."""
    if info["path"] == 2:   # one generated kernel per task (+ argmax if unfused)
        return info["n_tasks"] + (1 if want_am and info["n_tasks"] > 1 else 0)
    if info["path"] == 1:   # per transposed chunk: transpose + layered kernel
        chunk = max(1, info["chunk_samples"])
        rounds = (n + chunk - 1) // chunk
        # certified single pass: per round a gather, a hi/lo recompute and a
        # scatter (no-ops when every sample is certified)
        return 2 * rounds + (3 * rounds if info.get("certified") else 0)
    return 1


def run_ours(args):
    import torch
    import torch.distributed as dist

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if world > 1:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)

    from paper_conf_cgo_sommera022_b200.build import build
    if rank == 0:
        build()
    if world > 1:
        dist.barrier()
    import paper_conf_cgo_sommera022_b200 as spnb

    n_rank, scaling = samples_per_rank(args.config, world)
    if args.config in ("C4", "C5"):
        from spn_inputs import CONFIGS, config_graph
        from paper_conf_cgo_sommera022_b200.parallel import shard_range
        g = config_graph(args.config)
        n = n_rank
        lo = shard_range(CONFIGS_N(args.config), rank, world)[0] if scaling == "strong" \
            else rank * n
        xd = device_uniform(n, g.n_features, CONFIGS[args.config]["data_seed"], lo, dev)
        x = xd[:min(n, 1 << 20)].cpu().numpy()   # host copy of a bounded subset (e2e, oracle)
    else:
        g, x, n = make_workload(args.config, rank, args.marginal)
        xd = None
    G = spnb.Graph(g)
    t0 = time.perf_counter()
    P = spnb.Plan(G, device=local, samples_per_thread=args.K, block_threads=args.block,
                  tc_precision=args.tc_precision)
    prep_s = time.perf_counter() - t0
    info = P.info()
    if xd is None:
        xd = torch.from_numpy(x).to(dev)
    R = g.n_roots
    want_am = R > 1
    out = torch.empty((n, R), dtype=torch.float32, device=dev)
    am = torch.empty((n,), dtype=torch.int32, device=dev) if want_am else None
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
    st = torch.cuda.current_stream(dev)
    # strong scaling: every step ends with the gather of all ranks' results
    gather = scaling == "strong" and world > 1
    if gather:
        full_out = torch.empty((n * world, R), dtype=torch.float32, device=dev)
        full_am = torch.empty((n * world,), dtype=torch.int32, device=dev) if want_am else None

    def step():
        P.infer(xd, marginal=args.marginal, out=out, argmax=am, want_argmax=want_am, stream=st)

    def collect():
        # equal shards (10M / {1,2,4,8}): one all_gather_into_tensor each (NCCL)
        from paper_conf_cgo_sommera022_b200.parallel import gather_into
        gather_into(full_out, out)
        if want_am:
            gather_into(full_am, am)

    for _ in range(max(3, args.warmup)):
        flush.fill_(1)
        step()
        if gather:
            collect()
    torch.cuda.synchronize()
    clocks = ClockSampler(local)
    clocks.start()
    # keep the GPU busy ~0.5 s before the timed region so clocks settle
    t_end = time.perf_counter() + 0.5
    while time.perf_counter() < t_end:
        step()
        torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True),
            torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    for i in range(args.steps):
        flush.fill_(i & 0xff)
        evs[i][0].record(st)
        step()
        evs[i][1].record(st)
        if gather:
            collect()
        evs[i][2].record(st)
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    clk = clocks.stop()
    times = [a.elapsed_time(c) for a, b, c in evs]       # ms per step (infer + gather)
    gather_ms = [b.elapsed_time(c) for a, b, c in evs]
    tot_ms = sum(times)
    t = torch.tensor([tot_ms], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    tot_ms = float(t.item())
    n_job = CONFIGS_N(args.config) if scaling == "strong" else n * world
    value = n_job * args.steps / (tot_ms / 1e3)
    n_e2e = x.shape[0]

    # ---- end to end through the public host-buffer API (H2D + D2H inside) ----
    xh = torch.from_numpy(x).pin_memory()
    oh = torch.empty((n_e2e, R), dtype=torch.float32).pin_memory()
    amh = torch.empty((n_e2e,), dtype=torch.int32).pin_memory() if want_am else None
    P.infer_host(xh, marginal=args.marginal, out=oh, argmax=amh, want_argmax=want_am)
    e2e_steps = max(1, min(args.steps, 10))
    if world > 1:
        dist.barrier()
    t_e = time.perf_counter()
    for _ in range(e2e_steps):
        P.infer_host(xh, marginal=args.marginal, out=oh, argmax=amh, want_argmax=want_am)
    e2e_s = (time.perf_counter() - t_e) / e2e_steps
    te = torch.tensor([e2e_s], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(te, op=dist.ReduceOp.MAX)
    e2e_val = n_e2e * world / float(te.item())

    if rank == 0:
        peaks, src = _peaks()
        ms = tot_ms / args.steps
        rate = n / (ms / 1e3)                           # samples/s of one rank
        clock_mhz = peaks.get("sm_max_mhz", 1965.0)
        mufu_peak = 16 * 148 * clock_mhz * 1e6          # MUFU ops/s (16/clk/SM)
        fma_peak = 128 * 148 * clock_mhz * 1e6          # FP32 FMA lane-ops/s (128/clk/SM)
        mufu = info["mufu_per_sample"] * rate
        hbm = info["bytes_per_sample"] * rate / 1e9
        fma = info["fma_per_sample"] * rate
        tc = info["tc_flops_per_sample"] * rate
        tc_peak = peaks.get("bf16_tflops", 1590.0) * 1e12
        prof = os.path.join(ROOT, "profiles", f"ncu_{args.config}{'m' if args.marginal else ''}.json")
        traffic = None
        if os.path.exists(prof):
            with open(prof) as f:
                traffic = json.load(f).get("dram_bytes_per_launch")
        part = lambda a, p_, u: {"achieved": a, "peak": p_, "unit": u, "frac": a / p_}
        hbm_part = part(hbm, peaks["hbm_gbs"], "GB/s")
        mufu_part = part(mufu / 1e9, mufu_peak / 1e9, "Gop/s")
        # the metric's roofline: HBM or MUFU, whichever binds (time = max)
        hm = max(hbm_part["frac"], mufu_part["frac"])
        metric_roof = {"frac": hm, "binding": "hbm" if hbm_part["frac"] >= mufu_part["frac"]
                       else "mufu", "hbm": hbm_part, "mufu": mufu_part}
        peak_note = f"x 148 SMs x {clock_mhz:.0f} MHz (sm_max_mhz, {src})"
        if info["path"] in (0, 2) and hbm_part["frac"] >= mufu_part["frac"]:
            # e.g. C1 at 1e8 samples in linear space: one lg2 per sample, HBM binds
            roof = {"bound": "hbm", "achieved": hbm, "peak": peaks["hbm_gbs"], "unit": "GB/s",
                    "frac": hbm_part["frac"], "traffic": traffic,
                    "peak_source": f"hbm_gbs ({src})", "bytes_per_sample": info["bytes_per_sample"],
                    "value_space": "linear" if info.get("value_space") == 2 else "log2",
                    "hbm_mufu": metric_roof, "mufu": mufu_part}
        elif info["path"] in (0, 2):
            roof = {"bound": "alu", "pipe": "MUFU ex2/lg2 (16 op/clk/SM)",
                    "achieved": mufu / 1e9, "peak": mufu_peak / 1e9, "unit": "Gop/s",
                    "frac": mufu / mufu_peak, "traffic": traffic,
                    "peak_source": "16 MUFU/clk/SM " + peak_note,
                    "mufu_count": "sum over sums of the fan-in (n-1 ex2 + 1 lg2 per "
                                  "n-ary log-sum-exp)",
                    "hbm_mufu": metric_roof, "hbm": hbm_part}
        else:
            # layered path: the binding unit is the one with the highest
            # fraction -- FP32 FMA (FMA leaf layer + stage-2 contractions) or,
            # with the leaf layer on the tensor cores (leaf_tc), the tensor
            # pipe (algorithmic one-pass flops: leaf GEMMs + sum contractions)
            ltc = bool(info.get("leaf_tc"))
            fma_part = {"achieved": fma / 1e9, "peak": fma_peak / 1e9, "unit": "GFMA/s",
                        "frac": fma / fma_peak, "peak_source": "128 FMA/clk/SM " + peak_note,
                        "pipe": ("FP32 FMA (stage-2 contractions)" if ltc else
                                 "FP32 FMA (leaf layer + stage-2 contractions, 128 lanes/clk/SM)")}
            tc_part = {"achieved": tc / 1e12, "peak": tc_peak / 1e12, "unit": "TFLOP/s",
                       "frac": tc / tc_peak,
                       "flops": ("algorithmic, one pass: 2 I (2V+1) per leaf region (tensor-core "
                                 "leaves) + 2 na nb S per sum region" if ltc else
                                 "algorithmic, one pass (2 na nb S per sum region)"),
                       "passes_executed": {"leaf": 3 if ltc else 0, "sum": info["tc_passes"]},
                       "peak_source": f"bf16_tflops ({src}); f16 dense rate = bf16"}
            if tc_part["frac"] > fma_part["frac"]:
                roof = {"bound": "tensor", **tc_part, "traffic": traffic, "fma": fma_part,
                        "hbm_mufu": metric_roof}
            else:
                roof = {"bound": "alu", **fma_part, "traffic": traffic, "tensor": tc_part,
                        "hbm_mufu": metric_roof}
            roof["kernel"] = (f"layered v{info['layered_kernel']}" +
                              (", tensor-core leaves" if ltc else ""))
        # the oracle baseline is timed on rank 0 at N = 1 only (contract)
        cpu = cpu_baseline(g, x, args.marginal) if world == 1 else None
        line = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world,
                "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms,
                "higher_is_better": True, "scaling": scaling, "vs_baseline": None,
                "dtype": "f32", "data": ("synthetic (seeded ancestral samples)"
                                         if args.config not in ("C4", "C5") else
                                         "synthetic (counter-based U[0,1) per 65,536-sample chunk)"),
                "config": _config_dict(args, g, n, world, scaling) | {
                    "plan": {k: info[k] for k in ("path", "n_nodes", "n_tasks", "n_records",
                                                  "block_threads", "samples_per_thread",
                                                  "grid", "smem_bytes", "mufu_per_sample",
                                                  "fma_per_sample", "tc_flops_per_sample",
                                                  "max_stack", "kernel_regs", "ctas_per_sm",
                                                  "mufu_exec_per_sample", "compile_ms",
                                                  "chunk_samples", "layered_kernel",
                                                  "tc_passes", "leaf_tc", "certified")},
                    "prepare_s": prep_s,
                    "tc_precision": args.tc_precision},
                "roofline": roof, "cpu_baseline": cpu, "clocks": clk,
                "e2e": {"value": e2e_val, "unit": UNIT,
                        "h2d_bytes_per_step": int(x.nbytes),
                        "d2h_bytes_per_step": int(n_e2e * R * 4 + (n_e2e * 4 if want_am else 0)),
                        "samples_per_step": int(n_e2e),
                        "timing": "wall clock around the synchronous host-buffer call"},
                "gpu_launches": args.steps * launches_per_step(info, n, want_am),
                "step_ms": {"min": min(times), "median": statistics.median(times),
                            "max": max(times)}}
        if gather:
            line["gather_ms"] = {"median": statistics.median(gather_ms), "max": max(gather_ms),
                                 "what": "NCCL all_gather_into_tensor of logp [N/P, R] "
                                         "and argmax [N/P] (inside the timed step)"}
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--config", default="C5", choices=["C1", "C2", "C3", "C4", "C5"])
    ap.add_argument("--marginal", action="store_true")
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--K", type=int, default=0, help="samples per thread (0 = auto)")
    ap.add_argument("--block", type=int, default=0, help="threads per CTA (0 = auto)")
    ap.add_argument("--tc-precision", type=int, default=0,
                    help="layered path: 0 auto, 1 single f16 pass, 2 f16 hi/lo split")
    ap.add_argument("--samples", type=int, default=0,
                    help="override the config's sample count (e.g. C1 at 100000000)")
    args = ap.parse_args()
    if args.samples > 0:
        _N_OVERRIDE[args.config] = args.samples
    if args.impl == "reference":
        run_reference(args)
    else:
        run_ours(args)


if __name__ == "__main__":
    main()
