#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -q --timeout 300 -x -k "layered" > gpurun_out/pytest_layered.log 2>&1; echo "pytest_layered=$?" >> gpurun_out/status.txt
timeout 300 python scripts/profile_layered.py C4 1 > gpurun_out/prof_layered.log 2>&1; echo "prof_layered=$?" >> gpurun_out/status.txt
timeout 300 python scripts/profile_layered.py C4 3 > gpurun_out/prof_layered3.log 2>&1; echo "prof_layered3=$?" >> gpurun_out/status.txt
timeout 600 python bench.py --config C4 > gpurun_out/bench_c4.log 2>&1; echo "bench_c4=$?" >> gpurun_out/status.txt
