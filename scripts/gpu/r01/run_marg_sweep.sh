#!/bin/bash
# KS marginal launch sweep on C2 / C3: CTA size (registers per thread = 65536 / block)
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out; mkdir -p $O; : > $O/marg_sweep.jsonl
echo "# C2m auto (spill fallback to smaller CTAs)" >> $O/marg_sweep.jsonl
timeout 600 python bench.py --config C2 --marginal 2>>$O/marg_sweep.err | tail -1 >> $O/marg_sweep.jsonl
echo "# C3m auto" >> $O/marg_sweep.jsonl
timeout 900 python bench.py --config C3 --marginal 2>>$O/marg_sweep.err | tail -1 >> $O/marg_sweep.jsonl
timeout 600 python -m pytest tests -m gpu -q --timeout 600 -k "compiled or C2 or C3 or marginal" > $O/pytest_marg.log 2>&1; echo "pytest=$?" >> $O/marg_sweep.jsonl
for b in 768 640 512 384; do
  echo "# block $b" >> $O/marg_sweep.jsonl
  timeout 600 python bench.py --config C2 --marginal --block $b 2>>$O/marg_sweep.err | tail -1 >> $O/marg_sweep.jsonl
done
for b in 768 512; do
  echo "# C3 block $b" >> $O/marg_sweep.jsonl
  timeout 900 python bench.py --config C3 --marginal --block $b 2>>$O/marg_sweep.err | tail -1 >> $O/marg_sweep.jsonl
done
echo done >> $O/marg_sweep.jsonl
