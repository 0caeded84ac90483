#!/bin/bash
# layered kernel: serial MMA->epilogue with double-buffered weights (default) vs TMEM ping-pong overlap
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "layered or rat or c4 or C4" > $O/pytest_lay.log 2>&1; echo "pytest=$?" >> $O/status.txt
for ov in 0 1; do for p in 3 1; do
  SPNB_TMEM_OVERLAP=$ov timeout 300 python scripts/profile_layered.py C4 $p > $O/lay_ov${ov}_p$p.log 2>&1; echo "lay_ov${ov}_p$p=$?" >> $O/status.txt
done; done
timeout 900 python bench.py --config C4 > $O/bench_C4.log 2>&1; echo "bench_C4=$?" >> $O/status.txt
