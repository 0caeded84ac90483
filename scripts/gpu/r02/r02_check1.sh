#!/bin/bash
# r02 checkpoint: GPU tests, smoke, default bench (C5), C3 ncu capture + launch list
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/r02_check1; mkdir -p $O; : > $O/status.txt
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1; echo "build=$?" >> $O/status.txt
timeout 2400 python -m pytest tests -m gpu -q --timeout 1200 -x > $O/pytest_gpu.log 2>&1; echo "pytest=$?" >> $O/status.txt
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke=$?" >> $O/status.txt
timeout 1200 python bench.py > $O/bench_default.log 2>&1; echo "bench=$?" >> $O/status.txt
timeout 900 bash scripts/gpu/ncu_cap.sh $O/C3m spnb_t 64 2 python bench.py --config C3 --marginal --steps 1 --warmup 1; echo "ncu_C3=$?" >> $O/status.txt
echo done >> $O/status.txt
