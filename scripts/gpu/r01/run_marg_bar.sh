#!/bin/bash
# KS marginal (C2) barrier-spacing sweep at the default 1 x 768 launch
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out; mkdir -p $O; : > $O/marg_bar.jsonl
for b in 0 250 1000 2000; do
  echo "# SPNB_JIT_BAR=$b" >> $O/marg_bar.jsonl
  SPNB_JIT_BAR=$b timeout 300 python bench.py --marginal --steps 10 --warmup 3 2>>$O/marg_bar.err | tail -1 >> $O/marg_bar.jsonl
done
echo done >> $O/marg_bar.jsonl
