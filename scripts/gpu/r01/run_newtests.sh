#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out; mkdir -p $O
timeout 1500 python -m pytest tests/test_gpu_parity.py -q --timeout 900 --durations=8 -k "c3_full or c4_layered_marginal or c5_layered" > $O/pytest_new.log 2>&1; echo "pytest=$?" >> $O/status.txt
