#!/bin/bash
# v2 leaf loop variants (t-first ordering, 8 samples per leaf thread) A/B + parity
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/r02_leaf; mkdir -p $O; : > $O/status.txt
python -c "from paper_conf_cgo_sommera022_b200.build import build; build()" > $O/build.log 2>&1; echo "build=$?" >> $O/status.txt
run() { n=$1; shift; env "$@" timeout 200 python scripts/r2_check.py time1 > $O/time_$n.log 2>&1; echo "time_$n=$?" >> $O/status.txt; }
run a_default
run b_tfirst SPNB_LIB=variants/libspnb_tfirst.so
run c_spt8 SPNB_LIB=variants/libspnb_spt8.so
run d_tfirst_spt8 SPNB_LIB=variants/libspnb_tfirst_spt8.so
SPNB_LIB=variants/libspnb_tfirst.so timeout 600 python scripts/r2_check.py parity > $O/parity_tfirst.log 2>&1; echo "parity=$?" >> $O/status.txt
echo done >> $O/status.txt
