"""Build libspnb.so in-tree (sm_100a only).

nvcc compiles the kernel translation units (one per samples-per-thread K, in
parallel), g++ the host preparer / C ABI, and nvcc links everything with the
static CUDA runtime into ``paper_conf_cgo_sommera022_b200/libspnb.so``.
"""
from __future__ import annotations

import concurrent.futures as cf
import hashlib
import os
import shutil
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
INC = os.path.join(ROOT, "include")
BUILD = os.path.join(PKG, "_build")
LIB = os.path.join(PKG, "libspnb.so")

ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
NVCC_FLAGS = ARCH + ["-O3", "-std=c++17", "-lineinfo", "-Xcompiler", "-fPIC",
                     "-jtd", "10",  # dense switch -> one jump table (dag_eval.cuh)
                     "-I", CSRC, "-I", INC]
CXX_FLAGS = ["-O2", "-std=c++17", "-fPIC", "-Wall", "-I", CSRC, "-I", INC,
             "-I", "/usr/local/cuda/include"]

CU_SOURCES = ["dag_eval_k1.cu", "dag_eval_k2.cu", "dag_eval_k4.cu", "dag_eval_k8.cu",
              "rat_eval.cu", "rat2.cu", "argmax.cu"]
CXX_SOURCES = ["prepare.cpp", "layered.cpp", "codegen.cpp", "jit.cpp", "api.cpp"]
HEADERS = ["program.h", "dag_eval.cuh", "prepare.h", "layered.h", "codegen.h", "jit.h"]
# headers each CUDA translation unit includes (so editing host-side headers does
# not rebuild the slow interpreter objects)
CU_DEPS = {"rat_eval.cu": ["layered.h", "prepare.h", "program.h"],
           "rat2.cu": ["layered.h", "prepare.h", "program.h"], "argmax.cu": []}
CU_DEPS_DEFAULT = ["dag_eval.cuh", "program.h"]


def _nvcc():
    for c in (os.environ.get("NVCC"), "/usr/local/cuda/bin/nvcc", shutil.which("nvcc")):
        if c and os.path.exists(c):
            return c
    raise RuntimeError("nvcc not found")


def _digest(paths, extra):
    """Content hash of the sources/headers and the flags.  Absolute paths are
    left out so a tree copied elsewhere (the GPU box) reuses its objects."""
    h = hashlib.sha256()
    for p in paths:
        with open(p, "rb") as f:
            h.update(f.read())
    h.update(" ".join(a for a in extra if not os.path.isabs(a)).encode())
    return h.hexdigest()[:16]


def _compile(cmd, src, obj, stamp_key):
    stamp = obj + ".stamp"
    if os.path.exists(obj) and os.path.exists(stamp) and open(stamp).read() == stamp_key:
        return obj, False
    tmp = obj + f".tmp{os.getpid()}"
    r = subprocess.run(cmd + ["-c", src, "-o", tmp], capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError(f"compile failed: {src}\n{r.stdout}\n{r.stderr}")
    os.replace(tmp, obj)
    with open(stamp, "w") as f:
        f.write(stamp_key)
    return obj, True


def build(verbose: bool = False, jobs: int = 0) -> str:
    os.makedirs(BUILD, exist_ok=True)
    nvcc = _nvcc()
    hdrs = [os.path.join(CSRC, h) for h in HEADERS] + [os.path.join(INC, "spnb.h")]
    jobs = jobs or max(2, min(8, os.cpu_count() or 2))
    futs = []
    with cf.ThreadPoolExecutor(jobs) as ex:
        for s in CU_SOURCES:
            src = os.path.join(CSRC, s)
            obj = os.path.join(BUILD, s + ".o")
            deps = [os.path.join(CSRC, h) for h in CU_DEPS.get(s, CU_DEPS_DEFAULT)]
            key = _digest([src] + deps, NVCC_FLAGS)
            futs.append(ex.submit(_compile, [nvcc] + NVCC_FLAGS, src, obj, key))
        for s in CXX_SOURCES:
            src = os.path.join(CSRC, s)
            obj = os.path.join(BUILD, s + ".o")
            key = _digest([src] + hdrs, CXX_FLAGS)
            futs.append(ex.submit(_compile, ["g++"] + CXX_FLAGS, src, obj, key))
        objs = []
        changed = False
        for f in futs:
            o, ch = f.result()
            objs.append(o)
            changed |= ch
    if changed or not os.path.exists(LIB):
        tmp = LIB + f".tmp{os.getpid()}"
        cmd = [nvcc] + ARCH + ["-shared", "-cudart", "static", "-o", tmp] + objs
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode != 0:
            raise RuntimeError(f"link failed\n{r.stdout}\n{r.stderr}")
        os.replace(tmp, LIB)
        if verbose:
            print("built", LIB, file=sys.stderr)
    return LIB


if __name__ == "__main__":
    print(build(verbose=True))
