#!/bin/bash
# r02 checkpoint 6: LEAF_SPT 8 default: GPU tests, smoke, C5/C4 bench
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/r02_check6; mkdir -p $O; : > $O/status.txt
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1; echo "build=$?" >> $O/status.txt
timeout 2400 python -m pytest tests -m gpu -q --timeout 1200 > $O/pytest_gpu.log 2>&1; echo "pytest=$?" >> $O/status.txt
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke=$?" >> $O/status.txt
timeout 1200 python bench.py > $O/bench_C5.log 2>&1; echo "bench_C5=$?" >> $O/status.txt
timeout 900 python bench.py --config C4 > $O/bench_C4.log 2>&1; echo "bench_C4=$?" >> $O/status.txt
timeout 600 python scripts/r2_check.py parity > $O/parity.log 2>&1; echo "parity=$?" >> $O/status.txt
echo done >> $O/status.txt
