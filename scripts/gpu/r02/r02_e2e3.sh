#!/bin/bash
# grouped host pipeline with per-call (re)sized groups: host tests + C5 / C4 bench e2e
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/r02_e2e3; mkdir -p $O; : > $O/status.txt
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1; echo "build=$?" >> $O/status.txt
timeout 1500 python -m pytest tests -m gpu -q -k "host" --timeout 900 > $O/pytest_host.log 2>&1; echo "pytest=$?" >> $O/status.txt
timeout 1200 python bench.py > $O/bench_C5.log 2>&1; echo "bench_C5=$?" >> $O/status.txt
timeout 900 python bench.py --config C4 > $O/bench_C4.log 2>&1; echo "bench_C4=$?" >> $O/status.txt
echo done >> $O/status.txt
