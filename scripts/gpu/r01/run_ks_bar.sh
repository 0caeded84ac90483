#!/bin/bash
# KS: CTA-uniform grid-stride loop; optional CTA barriers in the straight-line body (icache locality)
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "compiled or c1 or c2 or C2 or ragged or c3" > $O/pytest_ks.log 2>&1; echo "pytest=$?" >> $O/status.txt
for b in 0 250 500 1000 2000; do
  SPNB_JIT_BAR=$b timeout 600 python bench.py --steps 10 > $O/bar_$b.log 2>&1; echo "bar_$b=$?" >> $O/status.txt
done
SPNB_JIT_BAR=1000 timeout 600 python bench.py --steps 10 --marginal > $O/bar_1000_m.log 2>&1; echo "bar_1000m=$?" >> $O/status.txt
SPNB_JIT_BAR=0 timeout 600 python bench.py --steps 10 --marginal > $O/bar_0_m.log 2>&1; echo "bar_0m=$?" >> $O/status.txt
