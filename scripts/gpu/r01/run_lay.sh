#!/bin/bash
# layered-kernel A/B: weight-group pipelining variants, precision, phase profile
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out; mkdir -p $O
for a in 0 1 2; do for p in 3 1; do
  SPNB_LAYERED_ATTEMPT=$a timeout 300 python scripts/profile_layered.py C4 $p > $O/lay_a${a}_p$p.log 2>&1; echo "lay_a${a}_p$p=$?" >> $O/status.txt
done; done
