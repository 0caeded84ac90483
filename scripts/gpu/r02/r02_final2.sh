#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/r02_final2; mkdir -p $O; : > $O/status.txt
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1; echo "build=$?" >> $O/status.txt
timeout 1200 python bench.py > $O/bench_C5.log 2>&1; echo "bench_C5=$?" >> $O/status.txt
for a in "C4" "C4 --marginal" "C2" "C2 --marginal" "C3 --marginal" "C1 --samples 100000000" "C1 --marginal --samples 100000000"; do
  n=$(echo $a | tr -d ' -' | sed 's/samples100000000/_1e8/'); timeout 900 python bench.py --config $a > $O/bench_$n.log 2>&1; echo "bench_$n=$?" >> $O/status.txt
done
timeout 900 python bench.py --impl reference > $O/bench_reference.log 2>&1; echo "bench_reference=$?" >> $O/status.txt
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 200 --csv --log-file $O/launches_C5.csv python bench.py --steps 1 --warmup 3 > $O/ncu_l_C5.log 2>&1; echo "ncul_C5=$?" >> $O/status.txt
SPNB_PROFILE=0 timeout 900 bash scripts/gpu/ncu_cap.sh $O/C5v2 rat2 0 1 python scripts/profile_layered.py C5 0; echo "ncu_C5=$?" >> $O/status.txt
echo done >> $O/status.txt
