#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/r02_v2l; mkdir -p $O; : > $O/status.txt
python -c "from paper_conf_cgo_sommera022_b200.build import build; build()" > $O/build.log 2>&1; echo "build=$?" >> $O/status.txt
timeout 600 python scripts/r2_check.py time > $O/time.log 2>&1; echo "time=$?" >> $O/status.txt
SPNB_PROFILE=0 bash scripts/gpu/ncu_cap.sh $O/C4v2 rat2 0 1 python scripts/profile_layered.py C4 1; echo "ncu=$?" >> $O/status.txt
echo done >> $O/status.txt
