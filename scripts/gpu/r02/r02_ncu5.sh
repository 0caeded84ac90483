#!/bin/bash
# ncu source-level capture of the v2 layered kernel on C5 (single f16 pass) + suspend-hint A/B
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/r02_ncu5; mkdir -p $O; : > $O/status.txt
python -c "from paper_conf_cgo_sommera022_b200.build import build; build()" > $O/build.log 2>&1; echo "build=$?" >> $O/status.txt
timeout 200 python scripts/r2_check.py time1 > $O/time_default.log 2>&1; echo "time_default=$?" >> $O/status.txt
SPNB_LIB=variants/libspnb_nohint.so timeout 200 python scripts/r2_check.py time1 > $O/time_nohint.log 2>&1; echo "time_nohint=$?" >> $O/status.txt
SPNB_PROFILE=0 bash scripts/gpu/ncu_cap.sh $O/C5v2 rat2 0 1 python scripts/profile_layered.py C5 1; echo "ncu=$?" >> $O/status.txt
echo done >> $O/status.txt
