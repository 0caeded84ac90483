#!/bin/bash
# tensor-core leaf layer (leaf_tc): hang check with the watchdog build, parity, timing vs FMA leaves, tests, profile
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/r02_ltc1; mkdir -p $O; : > $O/status.txt
python -c "from paper_conf_cgo_sommera022_b200.build import build; build()" > $O/build.log 2>&1; echo "build=$?" >> $O/status.txt
python scripts/build_variant.py wd -DR2_WATCHDOG >> $O/build.log 2>&1; echo "build_wd=$?" >> $O/status.txt
SPNB_LIB=variants/libspnb_wd.so timeout 90 python scripts/sanitize_cases.py v2 > $O/quick_wd.log 2>&1; echo "quick_wd=$?" >> $O/status.txt
if grep -q " ok " $O/quick_wd.log; then
  timeout 400 python scripts/r2_check.py ltc > $O/ltc_parity.log 2>&1; echo "ltc_parity=$?" >> $O/status.txt
  timeout 300 python scripts/r2_check.py ltctime > $O/ltc_time.log 2>&1; echo "ltc_time=$?" >> $O/status.txt
  SPNB_PROFILE=1 timeout 200 python scripts/profile_layered.py C4 0 > $O/prof_C4.log 2>&1; echo "prof=$?" >> $O/status.txt
  timeout 1200 python -m pytest tests -m gpu -q -x -k "layered or c4 or c5 or host_api" --timeout 900 > $O/pytest_layered.log 2>&1; echo "pytest=$?" >> $O/status.txt
fi
echo done >> $O/status.txt
