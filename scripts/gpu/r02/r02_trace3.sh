#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/${TRACE_OUT:-r02_trace3}; mkdir -p $O; : > $O/status.txt
python -c "from paper_conf_cgo_sommera022_b200.build import build; build()" > $O/build.log 2>&1; echo "build=$?" >> $O/status.txt
SPNB_LIB=${TRACE_LIB:-variants/libspnb_pgtrace.so} SPNB_PROFILE=1 timeout 300 python scripts/trace_layered.py C5 $O/trace_C5.npy > $O/trace_C5.log 2>&1; echo "trace5=$?" >> $O/status.txt
echo done >> $O/status.txt
