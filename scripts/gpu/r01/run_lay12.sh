#!/bin/bash
# layered: third weight buffer (ea rows computed by the epilogue threads, freeing smem)
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x --timeout 240 -k "layered or rat or c4 or C4 or c5" > $O/pytest_lay.log 2>&1; echo "pytest=$?" >> $O/status.txt
timeout 300 python scripts/profile_layered.py C4 3 > $O/lay_default.log 2>&1; echo "default=$?" >> $O/status.txt
SPNB_LAYERED_ATTEMPT=3 timeout 300 python scripts/profile_layered.py C4 3 > $O/lay_120x2.log 2>&1; echo "a3=$?" >> $O/status.txt
timeout 900 python bench.py --config C4 > $O/bench_C4.log 2>&1; echo "bench_C4=$?" >> $O/status.txt
