#!/bin/bash
# v2 timeline trace of CTA 0 (per-warp store trace, no atomics)
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/r02_trace2; mkdir -p $O; : > $O/status.txt
python -c "from paper_conf_cgo_sommera022_b200.build import build; build()" > $O/build.log 2>&1; echo "build=$?" >> $O/status.txt
SPNB_LIB=variants/libspnb_trace.so SPNB_PROFILE=1 timeout 300 python scripts/trace_layered.py C5 $O/trace_C5.npy > $O/trace_C5.log 2>&1; echo "trace5=$?" >> $O/status.txt
SPNB_LIB=variants/libspnb_trace.so SPNB_PROFILE=1 timeout 300 python scripts/r2_check.py time1 > $O/time_trace.log 2>&1; echo "time_trace=$?" >> $O/status.txt
echo done >> $O/status.txt
