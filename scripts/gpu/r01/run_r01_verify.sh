#!/bin/bash
# final verification on HEAD: GPU tests, smoke, default bench (C2 joint) and C2/C3 marginal
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out; mkdir -p $O; : > $O/verify_status.txt
timeout 1200 python -m pytest tests -m gpu -q --timeout 600 > $O/verify_pytest_gpu.log 2>&1; echo "pytest=$?" >> $O/verify_status.txt
timeout 600 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > $O/verify_smoke.log 2>&1; echo "smoke=$?" >> $O/verify_status.txt
timeout 600 python bench.py > $O/verify_bench_C2.log 2>&1; echo "bench=$?" >> $O/verify_status.txt
timeout 600 python bench.py --marginal > $O/verify_bench_C2m.log 2>&1; echo "bench_C2m=$?" >> $O/verify_status.txt
timeout 900 python bench.py --config C3 --marginal > $O/verify_bench_C3m.log 2>&1; echo "bench_C3m=$?" >> $O/verify_status.txt
echo done >> $O/verify_status.txt
