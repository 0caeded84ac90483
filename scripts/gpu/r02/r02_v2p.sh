#!/bin/bash
# A/B: 16-warp (4 leaf + 8 epilogue) vs 20-warp (8 leaf + 8 epilogue) v2 layouts
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/r02_v2p; mkdir -p $O; : > $O/status.txt
python -c "from paper_conf_cgo_sommera022_b200.build import build; build()" > $O/build.log 2>&1; echo "build=$?" >> $O/status.txt
SPNB_LIB=variants/libspnb_w20.so timeout 300 python scripts/r2_check.py parity > $O/parity_w20.log 2>&1; echo "parity_w20=$?" >> $O/status.txt
SPNB_LIB=variants/libspnb_w20.so SPNB_PROFILE=1 timeout 300 python scripts/profile_layered.py C4 1 > $O/prof_C4_w20.log 2>&1; echo "prof_w20=$?" >> $O/status.txt
SPNB_LIB=variants/libspnb_w20.so timeout 600 python scripts/r2_check.py time > $O/time_w20.log 2>&1; echo "time_w20=$?" >> $O/status.txt
timeout 600 python scripts/r2_check.py time > $O/time_w16.log 2>&1; echo "time_w16=$?" >> $O/status.txt
echo done >> $O/status.txt
