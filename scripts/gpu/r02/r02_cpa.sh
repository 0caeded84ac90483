#!/bin/bash
# v2: feature rows by cp.async instead of per-row bulk copies (A/B, parity, trace)
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/r02_cpa; mkdir -p $O; : > $O/status.txt
python -c "from paper_conf_cgo_sommera022_b200.build import build; build()" > $O/build.log 2>&1; echo "build=$?" >> $O/status.txt
run() { n=$1; shift; env "$@" timeout 200 python scripts/r2_check.py time1 > $O/time_$n.log 2>&1; echo "time_$n=$?" >> $O/status.txt; }
run default
run cpa SPNB_LIB=variants/libspnb_cpa.so
SPNB_LIB=variants/libspnb_cpa.so timeout 600 python scripts/r2_check.py parity > $O/parity_cpa.log 2>&1; echo "parity_cpa=$?" >> $O/status.txt
SPNB_LIB=variants/libspnb_cpatrace.so SPNB_PROFILE=1 timeout 300 python scripts/trace_layered.py C5 $O/trace_C5.npy > $O/trace_C5.log 2>&1; echo "trace5=$?" >> $O/status.txt
echo done >> $O/status.txt
