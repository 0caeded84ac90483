#!/bin/bash
# v2: per-group MMA issue (R2_MMA_PERGROUP) A/B, parity, trace
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/r02_pg; mkdir -p $O; : > $O/status.txt
python -c "from paper_conf_cgo_sommera022_b200.build import build; build()" > $O/build.log 2>&1; echo "build=$?" >> $O/status.txt
run() { n=$1; shift; env "$@" timeout 200 python scripts/r2_check.py time1 > $O/time_$n.log 2>&1; echo "time_$n=$?" >> $O/status.txt; }
run a_default
run b_pg SPNB_LIB=variants/libspnb_pg.so
run c_pg_r23 SPNB_LIB=variants/libspnb_pg.so SPNB_R2_RINGS=2,3
run d_pgup1 SPNB_LIB=variants/libspnb_pgup1.so
run e_pgup1_r23 SPNB_LIB=variants/libspnb_pgup1.so SPNB_R2_RINGS=2,3
SPNB_LIB=variants/libspnb_pg.so timeout 600 python scripts/r2_check.py parity > $O/parity_pg.log 2>&1; echo "parity=$?" >> $O/status.txt
SPNB_LIB=variants/libspnb_pgtrace.so SPNB_PROFILE=1 timeout 300 python scripts/trace_layered.py C5 $O/trace_C5.npy > $O/trace_C5.log 2>&1; echo "trace5=$?" >> $O/status.txt
echo done >> $O/status.txt
