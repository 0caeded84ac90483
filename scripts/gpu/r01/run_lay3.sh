#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out; mkdir -p $O
for w in 1 4 16; do for ov in 0 1; do
  SPNB_WREP=$w SPNB_TMEM_OVERLAP=$ov timeout 300 python scripts/profile_layered.py C4 3 > $O/lay_w${w}_ov$ov.log 2>&1; echo "lay_w${w}_ov$ov=$?" >> $O/status.txt
done; done
