#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out; mkdir -p $O
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/tmem_rate scripts/micro/tmem_rate.cu && timeout 120 /tmp/tmem_rate > $O/tmem_rate.log 2>&1; echo "tmem=$?" >> $O/status.txt
