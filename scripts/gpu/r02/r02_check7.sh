#!/bin/bash
# r02 checkpoint 7: LEAF_SPT 8 + LTC barrier counts fixed: GPU tests, smoke, then the SPT-8 A/B set
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/r02_check7; mkdir -p $O; : > $O/status.txt
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1; echo "build=$?" >> $O/status.txt
timeout 2400 python -m pytest tests -m gpu -q --timeout 600 > $O/pytest_gpu.log 2>&1; echo "pytest=$?" >> $O/status.txt
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke=$?" >> $O/status.txt
bash scripts/gpu/r02/r02_spt8ab.sh; cp gpurun_out/r02_spt8ab/* $O/ 2>/dev/null
echo done >> $O/status.txt
