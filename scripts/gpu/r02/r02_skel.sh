#!/bin/bash
# v2 synchronisation skeleton: all work knocked out (wrong results, timing only)
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/r02_skel; mkdir -p $O; : > $O/status.txt
python -c "from paper_conf_cgo_sommera022_b200.build import build; build()" > $O/build.log 2>&1; echo "build=$?" >> $O/status.txt
run() { n=$1; shift; env "$@" timeout 200 python scripts/r2_check.py time1 > $O/time_$n.log 2>&1; echo "time_$n=$?" >> $O/status.txt; }
run a_default
run b_skel SPNB_LIB=variants/libspnb_koskel.so
run c_komw SPNB_LIB=variants/libspnb_komw.so
run d_kocompute SPNB_LIB=variants/libspnb_kocompute.so
echo done >> $O/status.txt
