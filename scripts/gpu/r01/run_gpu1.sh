#!/bin/bash
# round-1 GPU session: smoke, gpu tests, bench, ncu captures
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,driver_version --format=csv > gpurun_out/smi.txt 2>&1
nproc > gpurun_out/nproc.txt; grep -m1 "model name" /proc/cpuinfo >> gpurun_out/nproc.txt
timeout 300 python __graft_entry__.py smoke > gpurun_out/smoke.log 2>&1; echo "smoke=$?" >> gpurun_out/status.txt
timeout 1200 python -m pytest tests -m gpu -q -x --timeout 600 > gpurun_out/pytest_gpu.log 2>&1; echo "pytest=$?" >> gpurun_out/status.txt
timeout 400 python bench.py > gpurun_out/bench.log 2>&1; echo "bench=$?" >> gpurun_out/status.txt
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 40 --csv --log-file gpurun_out/launches_c2.csv python bench.py --steps 5 --warmup 3 > gpurun_out/ncu_launch.log 2>&1; echo "ncu_launch=$?" >> gpurun_out/status.txt
timeout 900 ncu --set full --clock-control none --import-source on -k regex:dag_eval -s 6 -c 1 -o gpurun_out/prof_c2 python bench.py --steps 2 --warmup 3 > gpurun_out/ncu_full.log 2>&1; echo "ncu_full=$?" >> gpurun_out/status.txt
