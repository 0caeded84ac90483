#!/bin/bash
# compute-sanitizer memcheck / racecheck / synccheck on every kernel family (small inputs)
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/r02_sanitize; mkdir -p $O; : > $O/status.txt
python -c "from paper_conf_cgo_sommera022_b200.build import build; build()" > $O/build.log 2>&1; echo "build=$?" >> $O/status.txt
for c in v2 v1 interp compiled compiled_lin; do
  for t in memcheck racecheck synccheck; do
    timeout 600 compute-sanitizer --tool $t --error-exitcode 9 python scripts/sanitize_cases.py $c > $O/${c}_${t}.log 2>&1
    echo "${c}_${t}=$?" >> $O/status.txt
  done
done
echo done >> $O/status.txt
