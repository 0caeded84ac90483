#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out; mkdir -p $O
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/umma_rate scripts/micro/umma_rate.cu && timeout 120 /tmp/umma_rate > $O/umma_rate.log 2>&1; echo "umma=$?" >> $O/status.txt
