#!/bin/bash
# v2 ring-depth / UP-image-warp A/B (variants prebuilt in variants/)
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/r02_rings; mkdir -p $O; : > $O/status.txt
python -c "from paper_conf_cgo_sommera022_b200.build import build; build()" > $O/build.log 2>&1; echo "build=$?" >> $O/status.txt
run() { n=$1; shift; env "$@" timeout 200 python scripts/r2_check.py time1 > $O/time_$n.log 2>&1; echo "time_$n=$?" >> $O/status.txt; }
run default
run r23 SPNB_R2_RINGS=2,3
run up1 SPNB_LIB=variants/libspnb_upimg1.so
run up1_r23 SPNB_LIB=variants/libspnb_upimg1.so SPNB_R2_RINGS=2,3
run nab2_r33 SPNB_LIB=variants/libspnb_nab2.so SPNB_R2_RINGS=3,3
run nab2_r24 SPNB_LIB=variants/libspnb_nab2.so SPNB_R2_RINGS=2,4
run default2
SPNB_R2_RINGS=2,3 SPNB_PROFILE=1 timeout 200 python scripts/profile_layered.py C5 1 > $O/prof_r23.log 2>&1
echo done >> $O/status.txt
