#!/bin/bash
# 20-warp v2 layout with a balanced setmaxnreg budget (short timeouts: a hang costs little)
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/r02_v2q; mkdir -p $O; : > $O/status.txt
python -c "from paper_conf_cgo_sommera022_b200.build import build; build()" > $O/build.log 2>&1; echo "build=$?" >> $O/status.txt
SPNB_LIB=variants/libspnb_w20.so timeout 90 python scripts/sanitize_cases.py v2 > $O/quick_w20.log 2>&1; echo "quick_w20=$?" >> $O/status.txt
if grep -q "ok" $O/quick_w20.log; then
SPNB_LIB=variants/libspnb_w20.so timeout 300 python scripts/r2_check.py parity > $O/parity_w20.log 2>&1; echo "parity_w20=$?" >> $O/status.txt
SPNB_LIB=variants/libspnb_w20.so timeout 400 python scripts/r2_check.py time > $O/time_w20.log 2>&1; echo "time_w20=$?" >> $O/status.txt
fi
echo done >> $O/status.txt
