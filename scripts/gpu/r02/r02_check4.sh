#!/bin/bash
# r02 checkpoint 4: full GPU tests, smoke, bench lines (default C5, C4, C4m, C2, C2m, C3m), v2 racecheck with the slot fence
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/r02_check4; mkdir -p $O; : > $O/status.txt
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1; echo "build=$?" >> $O/status.txt
timeout 2400 python -m pytest tests -m gpu -q --timeout 1200 > $O/pytest_gpu.log 2>&1; echo "pytest=$?" >> $O/status.txt
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke=$?" >> $O/status.txt
timeout 1200 python bench.py > $O/bench_C5.log 2>&1; echo "bench_C5=$?" >> $O/status.txt
for a in "C4" "C4 --marginal" "C2" "C2 --marginal" "C3 --marginal"; do
  n=$(echo $a | tr -d ' -'); timeout 900 python bench.py --config $a > $O/bench_$n.log 2>&1; echo "bench_$n=$?" >> $O/status.txt
done
timeout 600 compute-sanitizer --tool racecheck --error-exitcode 9 python scripts/sanitize_cases.py v2 > $O/v2_racecheck.log 2>&1; echo "v2_racecheck=$?" >> $O/status.txt
echo done >> $O/status.txt
