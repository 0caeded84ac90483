#!/bin/bash
# FFMA2 leaf/epilogue in the layered kernel; KS at 3 CTAs/SM; FMA issue-rate microbenchmark; layered phase profile
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out; mkdir -p $O; rm -f $O/status.txt
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/fma_rate scripts/micro/fma_rate.cu && /tmp/fma_rate > $O/fma_rate.log 2>&1; echo "fma=$?" >> $O/status.txt
timeout 900 python -m pytest tests -m gpu -q -x --timeout 600 > $O/pytest_gpu.log 2>&1; echo "pytest=$?" >> $O/status.txt
timeout 600 python bench.py > $O/bench_C2.log 2>&1; echo "bench_C2=$?" >> $O/status.txt
timeout 900 python bench.py --config C4 > $O/bench_C4.log 2>&1; echo "bench_C4=$?" >> $O/status.txt
timeout 600 python scripts/profile_layered.py C4 3 > $O/prof_C4_p3.log 2>&1; echo "prof3=$?" >> $O/status.txt
timeout 600 python scripts/profile_layered.py C4 1 > $O/prof_C4_p1.log 2>&1; echo "prof1=$?" >> $O/status.txt
echo done >> $O/status.txt
