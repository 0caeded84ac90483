#!/bin/bash
# v2: epilogue-side slot release (one commit per group) A/B + parity
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/r02_rel; mkdir -p $O; : > $O/status.txt
python -c "from paper_conf_cgo_sommera022_b200.build import build; build()" > $O/build.log 2>&1; echo "build=$?" >> $O/status.txt
run() { n=$1; shift; env "$@" timeout 200 python scripts/r2_check.py time1 > $O/time_$n.log 2>&1; echo "time_$n=$?" >> $O/status.txt; }
run a_release
run b_norel SPNB_LIB=variants/libspnb_norel.so
timeout 600 python scripts/r2_check.py parity > $O/parity.log 2>&1; echo "parity=$?" >> $O/status.txt
timeout 1500 python -m pytest tests -m gpu -q -k "layered or c5 or c4 or host_api" --timeout 1200 > $O/pytest_layered.log 2>&1; echo "pytest=$?" >> $O/status.txt
echo done >> $O/status.txt
