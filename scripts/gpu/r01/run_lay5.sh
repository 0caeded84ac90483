#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "layered or rat or c4 or C4" > $O/pytest_lay.log 2>&1; echo "pytest=$?" >> $O/status.txt
timeout 300 python scripts/profile_layered.py C4 3 > $O/lay_base.log 2>&1; echo "base=$?" >> $O/status.txt
for u in u4 u8; do
  SPNB_LIB=variants/libspnb_$u.so timeout 300 python scripts/profile_layered.py C4 3 > $O/lay_$u.log 2>&1; echo "$u=$?" >> $O/status.txt
done
