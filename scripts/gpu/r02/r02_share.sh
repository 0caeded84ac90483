#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/r02_share; mkdir -p $O; : > $O/status.txt
python -c "from paper_conf_cgo_sommera022_b200.build import build; build()" > $O/build.log 2>&1; echo "build=$?" >> $O/status.txt
run() { n=$1; shift; env "$@" timeout 200 python scripts/r2_check.py time1 > $O/time_$n.log 2>&1; echo "time_$n=$?" >> $O/status.txt; }
run a_pgnh SPNB_LIB=variants/libspnb_pgnh.so
run b_share SPNB_LIB=variants/libspnb_share.so
run c_shareup1 SPNB_LIB=variants/libspnb_shareup1.so
run d_pgnh_r23 SPNB_LIB=variants/libspnb_pgnh.so SPNB_R2_RINGS=2,3
run e_share_r23 SPNB_LIB=variants/libspnb_share.so SPNB_R2_RINGS=2,3
echo done >> $O/status.txt
