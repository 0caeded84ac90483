#!/bin/bash
# r02 checkpoint 2: GPU tests, smoke, default bench (C5), config lines, ncu of the v2 kernel on C5
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/r02_check2; mkdir -p $O; : > $O/status.txt
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1; echo "build=$?" >> $O/status.txt
timeout 2400 python -m pytest tests -m gpu -q --timeout 1200 > $O/pytest_gpu.log 2>&1; echo "pytest=$?" >> $O/status.txt
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke=$?" >> $O/status.txt
timeout 1200 python bench.py > $O/bench_C5.log 2>&1; echo "bench_C5=$?" >> $O/status.txt
timeout 900 python bench.py --config C4 > $O/bench_C4.log 2>&1; echo "bench_C4=$?" >> $O/status.txt
timeout 900 python bench.py --config C4 --marginal > $O/bench_C4m.log 2>&1; echo "bench_C4m=$?" >> $O/status.txt
timeout 900 python bench.py --config C1 --samples 100000000 > $O/bench_C1_1e8.log 2>&1; echo "bench_C1_1e8=$?" >> $O/status.txt
timeout 900 python bench.py --config C1 --marginal --samples 100000000 > $O/bench_C1m_1e8.log 2>&1; echo "bench_C1m_1e8=$?" >> $O/status.txt
timeout 900 python bench.py --config C2 > $O/bench_C2.log 2>&1; echo "bench_C2=$?" >> $O/status.txt
timeout 900 python bench.py --config C3 --marginal > $O/bench_C3m.log 2>&1; echo "bench_C3m=$?" >> $O/status.txt
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 200 --csv --log-file $O/launches_C5.csv python bench.py --steps 1 --warmup 3 > $O/ncu_l_C5.log 2>&1; echo "ncul_C5=$?" >> $O/status.txt
SPNB_PROFILE=0 timeout 900 bash scripts/gpu/ncu_cap.sh $O/C5v2 rat2 0 1 python scripts/profile_layered.py C5 0; echo "ncu_C5=$?" >> $O/status.txt
echo done >> $O/status.txt
