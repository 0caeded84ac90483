#!/bin/bash
# layered kernel: grouped (a,b) parameter layout (LDS.128 pairs); full GPU suite
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out; mkdir -p $O
timeout 1200 python -m pytest tests -m gpu -q -x --timeout 600 > $O/pytest_gpu.log 2>&1; echo "pytest=$?" >> $O/status.txt
timeout 300 python scripts/profile_layered.py C4 3 > $O/lay_512.log 2>&1; echo "p512=$?" >> $O/status.txt
SPNB_RAT_THREADS=256 timeout 300 python scripts/profile_layered.py C4 3 > $O/lay_256.log 2>&1; echo "p256=$?" >> $O/status.txt
timeout 900 python bench.py --config C4 > $O/bench_C4.log 2>&1; echo "bench_C4=$?" >> $O/status.txt
