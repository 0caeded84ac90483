"""Build an experimental variant of libspnb.so with extra -D flags on the
layered kernel translation units (A/B timing on the GPU box; load it with
SPNB_LIB=<path>).  Usage: build_variant.py NAME [-DFOO ...]"""
import os
import subprocess
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_cgo_sommera022_b200 import build as B  # noqa: E402

name, defs = sys.argv[1], sys.argv[2:]
B.build()
out_dir = os.path.join(B.ROOT, "variants")
os.makedirs(out_dir, exist_ok=True)
objs = []
for s in B.CU_SOURCES + B.CXX_SOURCES:
    obj = os.path.join(B.BUILD, s + ".o")
    if s in ("rat_eval.cu", "rat2.cu") and defs:
        vobj = os.path.join(out_dir, f"{s[:-3]}_{name}.o")
        subprocess.run([B._nvcc()] + B.NVCC_FLAGS + defs + ["-c", os.path.join(B.CSRC, s), "-o", vobj],
                       check=True)
        obj = vobj
    objs.append(obj)
lib = os.path.join(out_dir, f"libspnb_{name}.so")
subprocess.run([B._nvcc()] + B.ARCH + ["-shared", "-cudart", "static", "-o", lib] + objs, check=True)
print(lib)
