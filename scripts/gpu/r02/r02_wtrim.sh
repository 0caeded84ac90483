#!/bin/bash
# v2: trimmed weight copies (R2_WTRIM, default) vs full copies: A/B, parity, layered GPU tests
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/r02_wtrim; mkdir -p $O; : > $O/status.txt
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1; echo "build=$?" >> $O/status.txt
timeout 600 python scripts/r2_check.py parity > $O/parity.log 2>&1; echo "parity=$?" >> $O/status.txt
run() { n=$1; shift; env "$@" timeout 200 python scripts/r2_check.py time1 > $O/time_$n.log 2>&1; echo "time_$n=$?" >> $O/status.txt; }
run a_trim
run b_notrim SPNB_LIB=variants/libspnb_notrim.so
run c_trim2
timeout 1800 python -m pytest tests -m gpu -q -k "layered or c5 or c4 or host" --timeout 600 > $O/pytest_layered.log 2>&1; echo "pytest=$?" >> $O/status.txt
echo done >> $O/status.txt
