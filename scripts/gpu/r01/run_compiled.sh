#!/bin/bash
# compiled path: GPU tests, bench lines C1/C2/C2m/C3m, ncu launch list + full capture of the generated kernel
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out; mkdir -p $O
timeout 1500 python -m pytest tests -m gpu -q --timeout 600 --durations=15 > $O/pytest_gpu.log 2>&1; echo "pytest=$?" >> $O/status.txt
for c in C2 C1; do
  timeout 600 python bench.py --config $c > $O/bench_$c.log 2>&1; echo "bench_$c=$?" >> $O/status.txt
done
timeout 600 python bench.py --config C2 --marginal > $O/bench_C2m.log 2>&1; echo "bench_C2m=$?" >> $O/status.txt
timeout 900 python bench.py --config C3 --marginal > $O/bench_C3m.log 2>&1; echo "bench_C3m=$?" >> $O/status.txt
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 200 --csv --log-file $O/launches_C2.csv python bench.py --config C2 --steps 3 --warmup 3 > $O/ncu_l_C2.log 2>&1; echo "ncul_C2=$?" >> $O/status.txt
timeout 900 ncu --set full --clock-control none --import-source on -k regex:spnb_t0 -s 2 -c 1 -o $O/full_C2_compiled python bench.py --config C2 --steps 3 --warmup 3 > $O/ncu_f_C2.log 2>&1; echo "nculf_C2=$?" >> $O/status.txt
echo done >> $O/status.txt
