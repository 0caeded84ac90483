#!/bin/bash
# v2: mbarrier wait strategies (per-group MMA issue in all variants)
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/r02_wait; mkdir -p $O; : > $O/status.txt
python -c "from paper_conf_cgo_sommera022_b200.build import build; build()" > $O/build.log 2>&1; echo "build=$?" >> $O/status.txt
run() { n=$1; shift; env "$@" timeout 200 python scripts/r2_check.py time1 > $O/time_$n.log 2>&1; echo "time_$n=$?" >> $O/status.txt; }
run a_pg SPNB_LIB=variants/libspnb_pg.so
run b_pgs32 SPNB_LIB=variants/libspnb_pgs32.so
run c_pgs128 SPNB_LIB=variants/libspnb_pgs128.so
run d_pgnh SPNB_LIB=variants/libspnb_pgnh.so
echo done >> $O/status.txt
