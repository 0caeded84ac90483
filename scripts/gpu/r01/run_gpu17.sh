#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
for rep in 1 2; do for v in old leaf2 epi2 cur; do
  if [ $v = cur ]; then unset SPNB_LIB; else export SPNB_LIB=variants/libspnb_$v.so; fi
  echo "== $v rep $rep" >> gpurun_out/ab.log
  timeout 300 python scripts/profile_layered.py C4 1 2>&1 | tail -2 >> gpurun_out/ab.log
done; done
echo done >> gpurun_out/status.txt
