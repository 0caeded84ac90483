#!/bin/bash
# v2: double-buffered epilogue TMEM loads (R2_EPI_DB, default) vs batches of 2-4 sums (variant)
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/r02_db; mkdir -p $O; : > $O/status.txt
python -c "from paper_conf_cgo_sommera022_b200.build import build; build()" > $O/build.log 2>&1; echo "build=$?" >> $O/status.txt
run() { n=$1; shift; env "$@" timeout 200 python scripts/r2_check.py time1 > $O/time_$n.log 2>&1; echo "time_$n=$?" >> $O/status.txt; }
run a_db
run b_nodb SPNB_LIB=variants/libspnb_nodb.so
for v in ${EXTRA_VARIANTS}; do run c_$v SPNB_LIB=variants/libspnb_$v.so; done
timeout 600 python scripts/r2_check.py parity > $O/parity.log 2>&1; echo "parity=$?" >> $O/status.txt
echo done >> $O/status.txt
