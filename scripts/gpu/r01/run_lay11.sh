#!/bin/bash
# layered group loop: pair mode (two interleaved MMA chains) vs one group at a time
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "layered or rat or c4 or C4 or c5" > $O/pytest_lay.log 2>&1; echo "pytest=$?" >> $O/status.txt
timeout 300 python scripts/profile_layered.py C4 3 > $O/lay_pairs.log 2>&1; echo "pairs=$?" >> $O/status.txt
SPNB_LIB=variants/libspnb_nopairs.so timeout 300 python scripts/profile_layered.py C4 3 > $O/lay_nopairs.log 2>&1; echo "nopairs=$?" >> $O/status.txt
timeout 900 python bench.py --config C4 > $O/bench_C4.log 2>&1; echo "bench_C4=$?" >> $O/status.txt
