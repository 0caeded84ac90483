#!/bin/bash
# v2: two MMA-issuing warps (one per accumulator, R2_MMA2) A/B + parity (watchdog build)
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/r02_mma2; mkdir -p $O; : > $O/status.txt
python -c "from paper_conf_cgo_sommera022_b200.build import build; build()" > $O/build.log 2>&1; echo "build=$?" >> $O/status.txt
run() { n=$1; shift; env "$@" timeout 200 python scripts/r2_check.py time1 > $O/time_$n.log 2>&1; echo "time_$n=$?" >> $O/status.txt; }
SPNB_LIB=variants/libspnb_mma2.so timeout 300 python scripts/r2_check.py parity > $O/parity_mma2.log 2>&1; echo "parity=$?" >> $O/status.txt
run a_default
run b_mma2 SPNB_LIB=variants/libspnb_mma2.so
run c_default2
echo done >> $O/status.txt
