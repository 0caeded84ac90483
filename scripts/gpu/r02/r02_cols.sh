#!/bin/bash
# v2: wider TMEM batches for narrow (UP / root) sums (R2_EPI_COLS_NARROW) A/B + parity
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/r02_cols; mkdir -p $O; : > $O/status.txt
python -c "from paper_conf_cgo_sommera022_b200.build import build; build()" > $O/build.log 2>&1; echo "build=$?" >> $O/status.txt
run() { n=$1; shift; env "$@" timeout 200 python scripts/r2_check.py time1 > $O/time_$n.log 2>&1; echo "time_$n=$?" >> $O/status.txt; }
run a_default
run b_n120 SPNB_LIB=variants/libspnb_n120.so
run c_n100 SPNB_LIB=variants/libspnb_n100.so
run d_default2
SPNB_LIB=variants/libspnb_n120.so timeout 600 python scripts/r2_check.py parity > $O/parity_n120.log 2>&1; echo "parity=$?" >> $O/status.txt
echo done >> $O/status.txt
