#!/bin/bash
# A/B of v2 variants: leaf samples per thread (4/8) x epilogue group sharing (0/1); hang-checked first
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/r02_ab1; mkdir -p $O; : > $O/status.txt
python -c "from paper_conf_cgo_sommera022_b200.build import build; build()" > $O/build.log 2>&1; echo "build=$?" >> $O/status.txt
for v in default s8e0 s4e1 s4e0; do
  if [ $v = default ]; then L=""; else L="variants/libspnb_$v.so"; fi
  SPNB_LIB=$L timeout 60 python scripts/sanitize_cases.py v2 > $O/quick_$v.log 2>&1; echo "quick_$v=$?" >> $O/status.txt
  if grep -q " ok " $O/quick_$v.log; then
    SPNB_LIB=$L timeout 200 python scripts/r2_check.py time1 > $O/time_$v.log 2>&1; echo "time_$v=$?" >> $O/status.txt
  fi
done
SPNB_LIB= timeout 300 python scripts/r2_check.py parity > $O/parity_default.log 2>&1; echo "parity_default=$?" >> $O/status.txt
echo done >> $O/status.txt
