#!/bin/bash
# layered kernel: 512-thread (16-warp) variant vs 256
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "layered or rat or c4 or C4" > $O/pytest_lay.log 2>&1; echo "pytest=$?" >> $O/status.txt
timeout 300 python scripts/profile_layered.py C4 3 > $O/lay_512.log 2>&1; echo "p512=$?" >> $O/status.txt
SPNB_RAT_THREADS=256 timeout 300 python scripts/profile_layered.py C4 3 > $O/lay_256.log 2>&1; echo "p256=$?" >> $O/status.txt
timeout 300 python scripts/profile_layered.py C4 1 > $O/lay_512_p1.log 2>&1; echo "p512p1=$?" >> $O/status.txt
timeout 900 python bench.py --config C4 > $O/bench_C4.log 2>&1; echo "bench_C4=$?" >> $O/status.txt
