#!/bin/bash
# v2 kernel: small-shape parity, phase counters on C4/C5, ncu full capture on C4
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/r02_v2b; mkdir -p $O; : > $O/status.txt
python -c "from paper_conf_cgo_sommera022_b200.build import build; build()" > $O/build.log 2>&1; echo "build=$?" >> $O/status.txt
timeout 300 python scripts/r2_check.py parity > $O/parity.log 2>&1; echo "parity=$?" >> $O/status.txt
SPNB_PROFILE=1 timeout 300 python scripts/profile_layered.py C4 1 > $O/prof_C4.log 2>&1; echo "prof_C4=$?" >> $O/status.txt
SPNB_PROFILE=1 timeout 300 python scripts/profile_layered.py C5 1 > $O/prof_C5.log 2>&1; echo "prof_C5=$?" >> $O/status.txt
bash scripts/gpu/ncu_cap.sh $O/C4v2 rat2 0 1 python scripts/profile_layered.py C4 1; echo "ncu=$?" >> $O/status.txt
echo done >> $O/status.txt
