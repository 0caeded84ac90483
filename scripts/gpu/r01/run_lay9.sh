#!/bin/bash
# layered epilogue: all TMEM loads of a sum (or two) before one wait
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "layered or rat or c4 or C4" > $O/pytest_lay.log 2>&1; echo "pytest=$?" >> $O/status.txt
timeout 300 python scripts/profile_layered.py C4 3 > $O/lay_512.log 2>&1; echo "p512=$?" >> $O/status.txt
SPNB_RAT_THREADS=256 timeout 300 python scripts/profile_layered.py C4 3 > $O/lay_256.log 2>&1; echo "p256=$?" >> $O/status.txt
SPNB_LIB=variants/libspnb_sps2.so SPNB_RAT_THREADS=256 timeout 300 python scripts/profile_layered.py C4 3 > $O/lay_256_sps2.log 2>&1; echo "p256s2=$?" >> $O/status.txt
SPNB_TMEM_OVERLAP=1 timeout 300 python scripts/profile_layered.py C4 3 > $O/lay_512_ov1.log 2>&1; echo "p512ov=$?" >> $O/status.txt
