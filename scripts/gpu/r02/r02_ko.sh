#!/bin/bash
# critical-path knockouts of the v2 kernel (wrong results, timing only): leaf FMAs, stage-2 dots, MMAs, weight copies
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/r02_ko; mkdir -p $O; : > $O/status.txt
python -c "from paper_conf_cgo_sommera022_b200.build import build; build()" > $O/build.log 2>&1; echo "build=$?" >> $O/status.txt
for v in leaf epi mma w leafepi; do
  case $v in leaf) D="-DR2_KO_LEAF";; epi) D="-DR2_KO_EPI";; mma) D="-DR2_KO_MMA";; w) D="-DR2_KO_W";; leafepi) D="-DR2_KO_LEAF -DR2_KO_EPI";; esac
  python scripts/build_variant.py ko$v $D -DR2_WATCHDOG >> $O/build.log 2>&1; echo "build_$v=$?" >> $O/status.txt
done
timeout 200 python scripts/r2_check.py time1 > $O/time_default.log 2>&1; echo "time_default=$?" >> $O/status.txt
for v in leaf epi mma w leafepi; do
  SPNB_LIB=variants/libspnb_ko$v.so timeout 200 python scripts/r2_check.py time1 > $O/time_$v.log 2>&1; echo "time_$v=$?" >> $O/status.txt
  SPNB_LIB=variants/libspnb_ko$v.so SPNB_PROFILE=1 timeout 200 python scripts/profile_layered.py C4 1 > $O/prof_$v.log 2>&1
done
SPNB_PROFILE=1 timeout 200 python scripts/profile_layered.py C4 1 > $O/prof_default.log 2>&1
echo done >> $O/status.txt
