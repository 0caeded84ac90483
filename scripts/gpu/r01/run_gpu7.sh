#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -q --timeout 300 -x -k "layered" > gpurun_out/pytest_layered.log 2>&1; echo "pytest_layered=$?" >> gpurun_out/status.txt
timeout 600 python bench.py --config C4 --steps 5 --warmup 3 > gpurun_out/bench_c4.log 2>&1; echo "bench_c4=$?" >> gpurun_out/status.txt
timeout 600 python bench.py --config C4 --steps 5 --warmup 3 --tc-precision 1 > gpurun_out/bench_c4_p1.log 2>&1; echo "bench_c4_p1=$?" >> gpurun_out/status.txt
timeout 900 ncu --set full --clock-control none --import-source on -k regex:rat_eval -s 2 -c 1 -o gpurun_out/prof_c4_v2 python bench.py --config C4 --steps 1 --warmup 3 > gpurun_out/ncu_c4.log 2>&1; echo "ncu_c4=$?" >> gpurun_out/status.txt
