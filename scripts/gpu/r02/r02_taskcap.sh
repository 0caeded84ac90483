#!/bin/bash
# KS: speaker SPNs packed per kernel (SPNB_JIT_TASKCAP) on C3 marginal + C2 joint sanity
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/r02_taskcap; mkdir -p $O; : > $O/status.txt
python -c "from paper_conf_cgo_sommera022_b200.build import build; build()" > $O/build.log 2>&1; echo "build=$?" >> $O/status.txt
for c in 3000 6000 12000 25000; do
  SPNB_JIT_TASKCAP=$c timeout 900 python bench.py --config C3 --marginal --steps 10 --warmup 3 > $O/bench_C3m_$c.log 2>&1; echo "c3m_$c=$?" >> $O/status.txt
done
SPNB_JIT_TASKCAP=12000 timeout 900 python -m pytest tests -m gpu -q -k "c3 or compiled" --timeout 600 > $O/pytest_c3.log 2>&1; echo "pytest=$?" >> $O/status.txt
echo done >> $O/status.txt
