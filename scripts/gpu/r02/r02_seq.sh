#!/bin/bash
# v2: per-accumulator consecutive K-steps (default now) vs interleaved (variant)
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/r02_seq; mkdir -p $O; : > $O/status.txt
python -c "from paper_conf_cgo_sommera022_b200.build import build; build()" > $O/build.log 2>&1; echo "build=$?" >> $O/status.txt
run() { n=$1; shift; env "$@" timeout 200 python scripts/r2_check.py time1 > $O/time_$n.log 2>&1; echo "time_$n=$?" >> $O/status.txt; }
run seq
run interleave SPNB_LIB=variants/libspnb_il.so
timeout 600 python scripts/r2_check.py parity > $O/parity.log 2>&1; echo "parity=$?" >> $O/status.txt
SPNB_PROFILE=1 timeout 200 python scripts/profile_layered.py C5 1 > $O/prof_C5.log 2>&1
echo done >> $O/status.txt
