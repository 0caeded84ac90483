#!/bin/bash
# round-1 check after the compiled-path auto fix: GPU tests, smoke, KS launch sweep, C4/C5 layered bench lines, reference arm, C4 ncu
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out; mkdir -p $O; rm -f $O/status.txt
timeout 1200 python -m pytest tests -m gpu -q --timeout 600 --durations=15 > $O/pytest_gpu.log 2>&1; echo "pytest=$?" >> $O/status.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke=$?" >> $O/status.txt
for kb in "1 2" "1 3" "2 1"; do set -- $kb
  SPNB_JIT_K=$1 SPNB_JIT_MINB=$2 timeout 600 python bench.py --steps 10 > $O/sweep_K$1_B$2.log 2>&1; echo "sweep_K$1_B$2=$?" >> $O/status.txt
done
SPNB_JIT_K=1 SPNB_JIT_MINB=6 timeout 600 python bench.py --steps 10 --block 128 > $O/sweep_K1_B6_t128.log 2>&1; echo "sweep_t128=$?" >> $O/status.txt
for c in C4 C5; do
  timeout 900 python bench.py --config $c > $O/bench_$c.log 2>&1; echo "bench_$c=$?" >> $O/status.txt
done
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > $O/bench_ref.log 2>&1; echo "bench_ref=$?" >> $O/status.txt
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 300 --csv --log-file $O/launches_C4.csv python bench.py --config C4 --steps 3 --warmup 3 > $O/ncu_l_C4.log 2>&1; echo "ncul_C4=$?" >> $O/status.txt
timeout 900 ncu --set full --clock-control none --import-source on -k regex:rat -s 2 -c 1 -o $O/full_C4 python bench.py --config C4 --steps 3 --warmup 3 > $O/ncu_f_C4.log 2>&1; echo "nculf_C4=$?" >> $O/status.txt
echo done >> $O/status.txt
