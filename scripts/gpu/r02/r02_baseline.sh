#!/bin/bash
# r02 baseline: ncu full captures of the round-1 layered kernel on C5 and of the KS marginal kernels on C3
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/r02_base; mkdir -p $O; : > $O/status.txt
python -c "from paper_conf_cgo_sommera022_b200.build import build; build()" > $O/build.log 2>&1; echo "build=$?" >> $O/status.txt
timeout 900 ncu --set full --clock-control none --import-source on -k regex:rat_eval -s 1 -c 1 -o $O/full_C5_v1 python scripts/profile_layered.py C5 3 > $O/ncu_C5.log 2>&1; echo "ncu_C5=$?" >> $O/status.txt
timeout 900 ncu --set full --clock-control none --import-source on -k regex:spnb_t -s 64 -c 32 -o $O/full_C3m python bench.py --config C3 --marginal --steps 1 --warmup 1 > $O/ncu_C3.log 2>&1; echo "ncu_C3=$?" >> $O/status.txt
echo done >> $O/status.txt
