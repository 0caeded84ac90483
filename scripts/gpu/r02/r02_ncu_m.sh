#!/bin/bash
# ncu --set full of the marginal-query kernels the bench lines C2m / C4m time
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/r02_ncu_m; mkdir -p $O; : > $O/status.txt
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1; echo "build=$?" >> $O/status.txt
bash scripts/gpu/ncu_cap.sh $O/C2m spnb_t0_m 0 1 python bench.py --config C2 --marginal --steps 1 --warmup 1; echo "ncu_C2m=$?" >> $O/status.txt
bash scripts/gpu/ncu_cap.sh $O/C4m rat2 0 1 python bench.py --config C4 --marginal --steps 1 --warmup 1; echo "ncu_C4m=$?" >> $O/status.txt
echo done >> $O/status.txt
