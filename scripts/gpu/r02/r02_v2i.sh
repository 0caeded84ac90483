#!/bin/bash
# v2 kernel: parity, phase counters (1-pass and hi/lo), timings
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/r02_v2i; mkdir -p $O; : > $O/status.txt
python -c "from paper_conf_cgo_sommera022_b200.build import build; build()" > $O/build.log 2>&1; echo "build=$?" >> $O/status.txt
timeout 300 python scripts/r2_check.py parity > $O/parity.log 2>&1; echo "parity=$?" >> $O/status.txt
SPNB_PROFILE=1 timeout 300 python scripts/profile_layered.py C4 1 > $O/prof_C4.log 2>&1; echo "prof_C4=$?" >> $O/status.txt
SPNB_PROFILE=1 timeout 300 python scripts/profile_layered.py C4 2 > $O/prof_C4p2.log 2>&1; echo "prof_C4p2=$?" >> $O/status.txt
timeout 600 python scripts/r2_check.py time > $O/time.log 2>&1; echo "time=$?" >> $O/status.txt
echo done >> $O/status.txt
