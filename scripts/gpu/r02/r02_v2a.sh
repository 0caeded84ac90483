#!/bin/bash
# first GPU run of the v2 layered kernel: parity + timing (each step bounded)
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/r02_v2a; mkdir -p $O; : > $O/status.txt
python -c "from paper_conf_cgo_sommera022_b200.build import build; build()" > $O/build.log 2>&1; echo "build=$?" >> $O/status.txt
timeout 300 python scripts/r2_check.py parity > $O/parity.log 2>&1; echo "parity=$?" >> $O/status.txt
timeout 600 python scripts/r2_check.py time > $O/time.log 2>&1; echo "time=$?" >> $O/status.txt
nvidia-smi --query-gpu=index,clocks.sm,power.draw --format=csv >> $O/status.txt
echo done >> $O/status.txt
