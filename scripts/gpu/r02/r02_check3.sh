#!/bin/bash
# C1 at 1e8 with 4 samples/thread, v2 timing without the watchdog, GPU test subset, compute-sanitizer
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/r02_check3; mkdir -p $O; : > $O/status.txt
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1; echo "build=$?" >> $O/status.txt
timeout 600 python bench.py --config C1 --samples 100000000 > $O/bench_C1_1e8.log 2>&1; echo "bench_C1=$?" >> $O/status.txt
timeout 200 python scripts/r2_check.py time1 > $O/time1.log 2>&1; echo "time1=$?" >> $O/status.txt
timeout 900 python -m pytest tests -m gpu -q -k "c1 or value_space or layered or compiled" --timeout 600 > $O/pytest_subset.log 2>&1; echo "pytest=$?" >> $O/status.txt
bash scripts/gpu/r02/r02_sanitize.sh; cp -r gpurun_out/r02_sanitize $O/ 2>/dev/null
echo done >> $O/status.txt
