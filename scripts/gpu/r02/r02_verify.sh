#!/bin/bash
# r02 closing verification on HEAD: full GPU test suite + smoke
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/${VERIFY_OUT:-r02_verify}; mkdir -p $O; : > $O/status.txt
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1; echo "build=$?" >> $O/status.txt
timeout 2400 python -m pytest tests -m gpu -q --timeout 900 > $O/pytest_gpu.log 2>&1; echo "pytest=$?" >> $O/status.txt
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke=$?" >> $O/status.txt
echo done >> $O/status.txt
