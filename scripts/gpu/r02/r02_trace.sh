#!/bin/bash
# v2 timeline trace of CTA 0 (C5, C4) + TMEM-read knockouts
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/r02_trace; mkdir -p $O; : > $O/status.txt
python -c "from paper_conf_cgo_sommera022_b200.build import build; build()" > $O/build.log 2>&1; echo "build=$?" >> $O/status.txt
SPNB_LIB=variants/libspnb_trace.so SPNB_PROFILE=1 timeout 300 python scripts/trace_layered.py C5 $O/trace_C5.npy > $O/trace_C5.log 2>&1; echo "trace5=$?" >> $O/status.txt
SPNB_LIB=variants/libspnb_trace.so SPNB_PROFILE=1 timeout 300 python scripts/trace_layered.py C4 $O/trace_C4.npy > $O/trace_C4.log 2>&1; echo "trace4=$?" >> $O/status.txt
run() { n=$1; shift; env "$@" timeout 200 python scripts/r2_check.py time1 > $O/time_$n.log 2>&1; echo "time_$n=$?" >> $O/status.txt; }
run default
run kotld SPNB_LIB=variants/libspnb_kotld.so
run koall SPNB_LIB=variants/libspnb_koall.so
echo done >> $O/status.txt
