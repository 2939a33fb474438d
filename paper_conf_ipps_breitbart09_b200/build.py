"""Build libboids.so (the CUDA path) in-tree with nvcc for sm_100a.

    python -m paper_conf_ipps_breitbart09_b200.build [-v]

Flags: --fmad=false (DESIGN.md Appendix A: no contraction anywhere in the
library; the kernels also use explicit __f*_rn intrinsics), -lineinfo for ncu
source mapping, static cudart so the library does not depend on which CUDA
runtime torch loaded.  The forbidden flags of Appendix A (--use_fast_math,
-prec-div=false, -prec-sqrt=false, -ftz=true) are never passed.
"""
from __future__ import annotations

import glob
import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
CSRC = os.path.join(HERE, "csrc")
LIB = os.path.join(HERE, "libboids.so")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
FLAGS = ["-O3", "-std=c++17", "-lineinfo", "--fmad=false", "-Xcompiler", "-fPIC",
         "-Xcompiler", "-fvisibility=hidden", "-cudart", "static",
         "-I", os.path.join(ROOT, "include"), "-I", CSRC]
FORBIDDEN = ("--use_fast_math", "-use_fast_math", "-prec-div=false", "-prec-sqrt=false", "-ftz=true")


def sources():
    return sorted(glob.glob(os.path.join(CSRC, "*.cu")))


def deps():
    return sources() + glob.glob(os.path.join(CSRC, "*.cuh")) + glob.glob(os.path.join(CSRC, "*.h")) + \
        [os.path.join(ROOT, "include", "boids.h"), os.path.abspath(__file__)]


def stale() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    return any(os.path.getmtime(d) > t for d in deps())


def build(verbose: bool = False, force: bool = False) -> str:
    if not force and not stale():
        return LIB
    assert not any(f in FORBIDDEN for f in FLAGS)
    objdir = os.path.join(HERE, "build")
    os.makedirs(objdir, exist_ok=True)
    objs = []
    extra = ["-Xptxas", "-v"] if verbose else []
    if os.environ.get("BOIDS_CHECKS") == "1":  # device bounds checks (internal.h BOIDS_CHECK); test builds only
        extra += ["-DBOIDS_CHECKS"]
    procs = []
    for src in sources():
        obj = os.path.join(objdir, os.path.basename(src) + ".o")
        cmd = [NVCC, *ARCH, *FLAGS, *extra, "-c", src, "-o", obj]
        procs.append((cmd, subprocess.Popen(cmd, stdout=subprocess.PIPE, stderr=subprocess.STDOUT, text=True)))
        objs.append(obj)
    failed = False
    for cmd, p in procs:
        out, _ = p.communicate()
        if out and (verbose or p.returncode):
            sys.stderr.write(out)
        if p.returncode:
            sys.stderr.write("FAILED: " + " ".join(cmd) + "\n")
            failed = True
    if failed:
        raise RuntimeError("nvcc failed")
    tmp = LIB + f".tmp{os.getpid()}"
    subprocess.check_call([NVCC, *ARCH, "-shared", "-cudart", "static", "-o", tmp, *objs])
    os.replace(tmp, LIB)
    return LIB


if __name__ == "__main__":
    build(verbose="-v" in sys.argv, force=True)
    print(LIB)
