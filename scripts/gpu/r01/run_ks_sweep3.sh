#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out; mkdir -p $O
for cfg in "1024 1 500" "768 1 250" "768 1 1000" "640 1 500" "896 1 500"; do set -- $cfg
  SPNB_JIT_BAR=$3 SPNB_JIT_MINB=$2 timeout 600 python bench.py --steps 10 --block $1 > $O/sw_$1_$3.log 2>&1; echo "sw_$1_$3=$?" >> $O/status.txt
  SPNB_JIT_BAR=$3 SPNB_JIT_MINB=$2 timeout 600 python bench.py --steps 10 --block $1 --marginal > $O/sw_$1_$3_m.log 2>&1; echo "sw_$1_$3_m=$?" >> $O/status.txt
done
SPNB_JIT_MINB=1 timeout 900 python bench.py --config C3 --marginal --steps 5 --block 768 > $O/c3m_768.log 2>&1; echo "c3m=$?" >> $O/status.txt
