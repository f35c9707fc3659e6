"""Build the in-tree CUDA library libfd.so (sm_100a) with nvcc.  No JIT, no torch extension:
the C ABI in include/fd.h is the boundary and this file only compiles it."""
from __future__ import annotations

import os
import shutil
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
OUT = os.path.join(PKG, "libfd.so")
OBJ = os.path.join(PKG, "build")
SOURCES = ["k_integral.cu", "k_cascade.cu", "k_cascade_ws.cu", "k_output.cu", "fd_api.cpp"]
HEADERS = [os.path.join(CSRC, "fd_internal.h"), os.path.join(CSRC, "k_common.cuh"), os.path.join(ROOT, "include", "fd.h")]
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
# --fmad=false: no FMA contraction anywhere (the kernels also use explicit __fmul_rn/__fadd_rn)
NVFLAGS = ["-O3", "-lineinfo", "-std=c++17", "--fmad=false", "-Xcompiler", "-fPIC,-O2", "-I", os.path.join(ROOT, "include")]


def _nvcc() -> str:
    for c in (os.environ.get("NVCC"), "/usr/local/cuda/bin/nvcc", shutil.which("nvcc")):
        if c and os.path.exists(c):
            return c
    raise RuntimeError("nvcc not found")


def build(force: bool = False, verbose: bool = False, variant: str = "") -> str:
    """variant "timing" builds libfd_timing.so with -DFD_K2_TIMING (K2 phase counters)."""
    nvcc = _nvcc()
    if variant:
        return _build_variant(nvcc, variant, verbose)
    os.makedirs(OBJ, exist_ok=True)
    hdr_t = max(os.path.getmtime(h) for h in HEADERS)
    objs = []
    rebuilt = False
    for src in SOURCES:
        s = os.path.join(CSRC, src)
        o = os.path.join(OBJ, src + ".o")
        objs.append(o)
        if force or not os.path.exists(o) or os.path.getmtime(o) < max(os.path.getmtime(s), hdr_t):
            cmd = [nvcc, *ARCH, *NVFLAGS, "-c", s, "-o", o]
            if verbose:
                print(" ".join(cmd), file=sys.stderr)
            subprocess.check_call(cmd)
            rebuilt = True
    if rebuilt or not os.path.exists(OUT) or os.path.getmtime(OUT) < max(os.path.getmtime(o) for o in objs):
        tmp = OUT + ".tmp"
        subprocess.check_call([nvcc, *ARCH, "-shared", "-cudart", "static", "-o", tmp, *objs, "-ldl"])
        os.replace(tmp, OUT)
    return OUT


def _build_variant(nvcc: str, variant: str, verbose: bool) -> str:
    defs = {"timing": ["-DFD_K2_TIMING"]}[variant]
    odir = os.path.join(OBJ, variant)
    os.makedirs(odir, exist_ok=True)
    objs = []
    for src in SOURCES:
        o = os.path.join(odir, src + ".o")
        cmd = [nvcc, *ARCH, *NVFLAGS, *defs, "-c", os.path.join(CSRC, src), "-o", o]
        if verbose:
            print(" ".join(cmd), file=sys.stderr)
        subprocess.check_call(cmd)
        objs.append(o)
    out = os.path.join(PKG, f"libfd_{variant}.so")
    subprocess.check_call([nvcc, *ARCH, "-shared", "-cudart", "static", "-o", out, *objs, "-ldl"])
    return out


if __name__ == "__main__":
    v = [a.split("=", 1)[1] for a in sys.argv if a.startswith("--variant=")]
    print(build(force="--force" in sys.argv, verbose=True, variant=v[0] if v else ""))
