#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
timeout 300 python scripts/sweep.py --combos 2:768,2:704,2:640,2:512,4:384 > gpurun_out/sweep_c2.log 2>&1; echo "sweep=$?" >> gpurun_out/status.txt
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -q --timeout 300 -x -k "samples_per_thread or layered_rat_small" > gpurun_out/pytest_gpu.log 2>&1; echo "pytest=$?" >> gpurun_out/status.txt
timeout 600 python bench.py --config C4 --steps 5 --warmup 3 --tc-precision 1 > gpurun_out/bench_c4_p1.log 2>&1; echo "bench_c4_p1=$?" >> gpurun_out/status.txt
