"""Build ``libfsgc.so`` (the C-ABI library) in-tree with nvcc for sm_100a.

    python paper_conf_sc_bradleyab25_b200/build.py          # incremental
    python paper_conf_sc_bradleyab25_b200/build.py --force
(run as a script: importing the package would try to load the library)

Objects go to ``paper_conf_sc_bradleyab25_b200/_build/``; the shared library to
``paper_conf_sc_bradleyab25_b200/libfsgc.so`` (git-ignored, travels to the GPU
box with gpurun).
"""
import os
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
CSRC = os.path.join(PKG, "csrc")
OUT = os.path.join(PKG, "_build")
LIB = os.path.join(PKG, "libfsgc.so")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
COMMON = ["-O3", "-std=c++17", "-lineinfo", "-Xcompiler", "-fPIC,-O3", "-I", CSRC]

SOURCES = ["pattern.cpp", "graph.cu", "count.cu"]
HEADERS = ["internal.h", "devbuf.cuh", "u128.cuh", "fc.cuh", "listing.cuh"]


def _newer(src, dst):
    return not os.path.exists(dst) or os.path.getmtime(src) > os.path.getmtime(dst)


def build(force=False, verbose=False):
    os.makedirs(OUT, exist_ok=True)
    hdr_paths = [os.path.join(CSRC, h) for h in HEADERS]
    hdr_paths.append(os.path.join(os.path.dirname(PKG), "include", "fsgc.h"))
    objs = []
    for s in SOURCES:
        src = os.path.join(CSRC, s)
        obj = os.path.join(OUT, s + ".o")
        objs.append(obj)
        stale = force or _newer(src, obj) or any(_newer(h, obj) for h in hdr_paths)
        if not stale:
            continue
        cmd = [NVCC] + ARCH + COMMON + ["-c", src, "-o", obj]
        if s.endswith(".cu"):
            cmd += ["-Xptxas", "-v"] if verbose else []
        else:
            cmd = [NVCC, "-x", "cu"] + ARCH + COMMON + ["-c", src, "-o", obj]
        if verbose:
            print(" ".join(cmd), flush=True)
        subprocess.run(cmd, check=True)
    if force or any(_newer(o, LIB) for o in objs):
        cmd = [NVCC] + ARCH + ["-shared", "-cudart", "static", "-Xcompiler", "-fPIC", "-o", LIB] + objs
        if verbose:
            print(" ".join(cmd), flush=True)
        subprocess.run(cmd, check=True)
    return LIB


if __name__ == "__main__":
    build(force="--force" in sys.argv, verbose=True)
