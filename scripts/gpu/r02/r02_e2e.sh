#!/bin/bash
# host pipeline of certified layered plans grouped (one certification round per group): probe + tests + bench e2e
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/${E2E_OUT:-r02_e2e}; mkdir -p $O; : > $O/status.txt
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1; echo "build=$?" >> $O/status.txt
timeout 600 python scripts/e2e_probe.py C5 > $O/probe_C5.log 2>&1; echo "probe=$?" >> $O/status.txt
timeout 1500 python -m pytest tests -m gpu -q -k "host" --timeout 1200 > $O/pytest_host.log 2>&1; echo "pytest=$?" >> $O/status.txt
timeout 1200 python bench.py > $O/bench_C5.log 2>&1; echo "bench_C5=$?" >> $O/status.txt
timeout 900 python bench.py --config C4 > $O/bench_C4.log 2>&1; echo "bench_C4=$?" >> $O/status.txt
echo done >> $O/status.txt
