#!/bin/bash
# ncu_cap.sh <out_prefix> <kernel_regex> <skip> <count> <cmd...>
# full ncu capture to /tmp, then raw + source pages as CSV under gpurun_out
# (the .ncu-rep itself is kept only when small)
pre=$1; kre=$2; skip=$3; cnt=$4; shift 4
rep=/tmp/$(basename $pre).ncu-rep
timeout 1200 ncu --set full --clock-control none --import-source on -k "regex:$kre" -s $skip -c $cnt -o ${rep%.ncu-rep} "$@" > ${pre}_ncu.log 2>&1
echo "ncu_rc=$?" >> ${pre}_ncu.log
ncu -i $rep --page raw --csv > ${pre}_raw.csv 2>>${pre}_ncu.log
ncu -i $rep --page source --csv > ${pre}_source.csv 2>>${pre}_ncu.log
ncu -i $rep --page details --csv > ${pre}_details.csv 2>>${pre}_ncu.log
sz=$(stat -c %s $rep 2>/dev/null || echo 0)
if [ "$sz" -lt 20000000 ]; then cp $rep ${pre}.ncu-rep; fi
