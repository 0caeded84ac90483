#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -q --timeout 600 -x > gpurun_out/pytest_gpu.log 2>&1; echo "pytest=$?" >> gpurun_out/status.txt
timeout 300 python scripts/sweep.py --combos 4:384,4:256,2:512,4:128 > gpurun_out/sweep_c2.log 2>&1; echo "sweep=$?" >> gpurun_out/status.txt
timeout 400 python bench.py > gpurun_out/bench.log 2>&1; echo "bench=$?" >> gpurun_out/status.txt
timeout 900 ncu --set full --clock-control none --import-source on -k regex:dag_eval -s 6 -c 1 -o gpurun_out/prof_c2_v3 python bench.py --steps 2 --warmup 3 > gpurun_out/ncu_full.log 2>&1; echo "ncu_full=$?" >> gpurun_out/status.txt
