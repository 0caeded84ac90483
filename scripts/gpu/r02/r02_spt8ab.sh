#!/bin/bash
# v2 with LEAF_SPT 8: ring depths, UP-image warp, wait hint, pair-wise MMA issue (A/B)
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/r02_spt8ab; mkdir -p $O; : > $O/status.txt
python -c "from paper_conf_cgo_sommera022_b200.build import build; build()" > $O/build.log 2>&1; echo "build=$?" >> $O/status.txt
run() { n=$1; shift; env "$@" timeout 200 python scripts/r2_check.py time1 > $O/time_$n.log 2>&1; echo "time_$n=$?" >> $O/status.txt; }
run a_default
run b_r23 SPNB_R2_RINGS=2,3
run c_nab2_r33 SPNB_LIB=variants/libspnb_nab2.so SPNB_R2_RINGS=3,3
run d_nab2_r24 SPNB_LIB=variants/libspnb_nab2.so SPNB_R2_RINGS=2,4
run e_up1 SPNB_LIB=variants/libspnb_up1.so
run f_hint SPNB_LIB=variants/libspnb_hint.so
run g_pair SPNB_LIB=variants/libspnb_pair.so
run h_default2
echo done >> $O/status.txt
