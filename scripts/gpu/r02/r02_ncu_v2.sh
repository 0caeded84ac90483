#!/bin/bash
# ncu source-level capture of the v2 layered kernel on C4 (single f16 pass)
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/r02_ncu_v2f; mkdir -p $O; : > $O/status.txt
python -c "from paper_conf_cgo_sommera022_b200.build import build; build()" > $O/build.log 2>&1; echo "build=$?" >> $O/status.txt
bash scripts/gpu/ncu_cap.sh $O/C4v2 rat2 0 1 python scripts/profile_layered.py C4 1; echo "ncu=$?" >> $O/status.txt
echo done >> $O/status.txt
