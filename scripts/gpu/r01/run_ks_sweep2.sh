#!/bin/bash
# KS launch sweep with the barrier-synchronised body
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out; mkdir -p $O
for cfg in "256 3" "512 1" "384 2" "128 6" "768 1"; do set -- $cfg
  SPNB_JIT_MINB=$2 timeout 600 python bench.py --steps 10 --block $1 > $O/sw_$1_$2.log 2>&1; echo "sw_$1_$2=$?" >> $O/status.txt
  SPNB_JIT_MINB=$2 timeout 600 python bench.py --steps 10 --block $1 --marginal > $O/sw_$1_$2_m.log 2>&1; echo "sw_$1_$2_m=$?" >> $O/status.txt
done
timeout 900 python bench.py --config C3 --marginal --steps 5 > $O/c3m.log 2>&1; echo "c3m=$?" >> $O/status.txt
