#!/bin/bash
# critical-path knockouts of the v2 kernel (variants prebuilt in variants/; wrong results, timing only)
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/r02_ko2; mkdir -p $O; : > $O/status.txt
python -c "from paper_conf_cgo_sommera022_b200.build import build; build()" > $O/build.log 2>&1; echo "build=$?" >> $O/status.txt
timeout 200 python scripts/r2_check.py time1 > $O/time_default.log 2>&1; echo "time_default=$?" >> $O/status.txt
SPNB_PROFILE=1 timeout 200 python scripts/profile_layered.py C5 1 > $O/prof_default_C5.log 2>&1
SPNB_PROFILE=1 timeout 200 python scripts/profile_layered.py C4 1 > $O/prof_default.log 2>&1
for v in leaf epi mma w leafepi; do
  SPNB_LIB=variants/libspnb_ko$v.so timeout 200 python scripts/r2_check.py time1 > $O/time_$v.log 2>&1; echo "time_$v=$?" >> $O/status.txt
  SPNB_LIB=variants/libspnb_ko$v.so SPNB_PROFILE=1 timeout 200 python scripts/profile_layered.py C4 1 > $O/prof_$v.log 2>&1
done
echo done >> $O/status.txt
