#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
timeout 300 python scripts/sweep.py --combos 2:768,2:704,1:1024,1:768,4:384 > gpurun_out/sweep_c2.log 2>&1; echo "sweep=$?" >> gpurun_out/status.txt
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q --timeout 300 -x -k "c1 or c2 or c3 or tiny or shard or host or empty" > gpurun_out/pytest_gpu.log 2>&1; echo "pytest=$?" >> gpurun_out/status.txt
timeout 400 python bench.py > gpurun_out/bench.log 2>&1; echo "bench=$?" >> gpurun_out/status.txt
timeout 900 ncu --set full --clock-control none --import-source on -k regex:dag_eval -s 6 -c 1 -o gpurun_out/prof_c2_v6 python bench.py --steps 2 --warmup 3 > gpurun_out/ncu_full.log 2>&1; echo "ncu_full=$?" >> gpurun_out/status.txt
