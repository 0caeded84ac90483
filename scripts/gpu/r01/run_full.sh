#!/bin/bash
# Full round check: GPU tests, smoke, bench lines for every config, ncu launch lists + one full capture.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out; mkdir -p $O
timeout 900 python -m pytest tests -m gpu -q --timeout 400 > $O/pytest_gpu.log 2>&1; echo "pytest=$?" >> $O/status.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke=$?" >> $O/status.txt
for c in C1 C2 C4 C5; do
  timeout 600 python bench.py --config $c > $O/bench_$c.log 2>&1; echo "bench_$c=$?" >> $O/status.txt
done
timeout 600 python bench.py --config C2 --marginal > $O/bench_C2m.log 2>&1; echo "bench_C2m=$?" >> $O/status.txt
timeout 600 python bench.py --config C3 --marginal > $O/bench_C3m.log 2>&1; echo "bench_C3m=$?" >> $O/status.txt
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > $O/bench_ref.log 2>&1; echo "bench_ref=$?" >> $O/status.txt
for c in C2 C4; do
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 200 --csv --log-file $O/launches_$c.csv python bench.py --config $c --steps 3 --warmup 3 > $O/ncu_l_$c.log 2>&1; echo "ncul_$c=$?" >> $O/status.txt
done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:dag_eval -s 2 -c 1 -o $O/full_C2 python bench.py --config C2 --steps 3 --warmup 3 > $O/ncu_f_C2.log 2>&1; echo "nculf_C2=$?" >> $O/status.txt
timeout 900 ncu --set full --clock-control none --import-source on -k regex:rat -s 1 -c 1 -o $O/full_C4 python bench.py --config C4 --steps 3 --warmup 3 > $O/ncu_f_C4.log 2>&1; echo "nculf_C4=$?" >> $O/status.txt
echo done >> $O/status.txt
