#!/bin/bash
# r01 closing evidence: GPU tests, smoke, bench lines (default = C2 joint), marginal configs after the per-variant launch-bound fix, C4/C5, reference arm
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out; mkdir -p $O
timeout 900 python -m pytest tests -m gpu -q --timeout 400 > $O/pytest_gpu.log 2>&1; echo "pytest=$?" >> $O/status.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke=$?" >> $O/status.txt
timeout 600 python bench.py > $O/bench_default.log 2>&1; echo "bench_default=$?" >> $O/status.txt
timeout 600 python bench.py --config C2 --marginal > $O/bench_C2m.log 2>&1; echo "bench_C2m=$?" >> $O/status.txt
timeout 900 python bench.py --config C3 --marginal > $O/bench_C3m.log 2>&1; echo "bench_C3m=$?" >> $O/status.txt
timeout 600 python bench.py --config C1 --marginal > $O/bench_C1m.log 2>&1; echo "bench_C1m=$?" >> $O/status.txt
timeout 600 python bench.py --config C4 --marginal > $O/bench_C4m.log 2>&1; echo "bench_C4m=$?" >> $O/status.txt
echo done >> $O/status.txt
