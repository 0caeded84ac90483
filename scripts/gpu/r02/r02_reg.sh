#!/bin/bash
# v2: setmaxnreg split (leaf / producer-MMA registers) A/B
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/r02_reg; mkdir -p $O; : > $O/status.txt
python -c "from paper_conf_cgo_sommera022_b200.build import build; build()" > $O/build.log 2>&1; echo "build=$?" >> $O/status.txt
run() { n=$1; shift; env "$@" timeout 200 python scripts/r2_check.py time1 > $O/time_$n.log 2>&1; echo "time_$n=$?" >> $O/status.txt; }
run a_default
run b_reg144 SPNB_LIB=variants/libspnb_reg144.so
run c_reg136 SPNB_LIB=variants/libspnb_reg136.so
run d_default2
echo done >> $O/status.txt
