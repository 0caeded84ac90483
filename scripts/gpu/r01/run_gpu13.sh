#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
timeout 300 python scripts/sweep.py --combos 2:768,2:704,4:384 > gpurun_out/sweep_c2.log 2>&1; echo "sweep=$?" >> gpurun_out/status.txt
timeout 300 python scripts/profile_layered.py C4 1 > gpurun_out/prof_layered.log 2>&1; echo "prof_layered=$?" >> gpurun_out/status.txt
timeout 1500 python -m pytest tests -m gpu -q --timeout 600 > gpurun_out/pytest_gpu.log 2>&1; echo "pytest=$?" >> gpurun_out/status.txt
timeout 400 python bench.py > gpurun_out/bench.log 2>&1; echo "bench=$?" >> gpurun_out/status.txt
timeout 600 python bench.py --config C4 --steps 5 --warmup 3 --tc-precision 1 > gpurun_out/bench_c4_p1.log 2>&1; echo "bench_c4_p1=$?" >> gpurun_out/status.txt
