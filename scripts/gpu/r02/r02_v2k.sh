#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/r02_v2k; mkdir -p $O; : > $O/status.txt
python -c "from paper_conf_cgo_sommera022_b200.build import build; build()" > $O/build.log 2>&1; echo "build=$?" >> $O/status.txt
timeout 300 python scripts/r2_check.py parity > $O/parity.log 2>&1; echo "parity=$?" >> $O/status.txt
timeout 600 python scripts/r2_check.py time > $O/time.log 2>&1; echo "time=$?" >> $O/status.txt
bash scripts/gpu/ncu_cap.sh $O/C4v2 rat2 0 1 python scripts/profile_layered.py C4 1; echo "ncu=$?" >> $O/status.txt
echo done >> $O/status.txt
