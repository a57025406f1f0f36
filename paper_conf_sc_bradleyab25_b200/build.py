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

# (source, object, extra flags): the counting kernels build once per
# accumulator class NP (count_np.cu -DFSGC_NPV=NP), all objects in parallel
SOURCES = [("pattern.cpp", "pattern.cpp.o", []), ("graph.cu", "graph.cu.o", []), ("count.cu", "count.cu.o", [])] + \
          [("count_np.cu", f"count_np{v}.cu.o", [f"-DFSGC_NPV={v}"]) for v in (1, 2, 4, 8, 16)]
HEADERS = ["internal.h", "devbuf.cuh", "u128.cuh", "fc.cuh", "listing.cuh", "count_dev.cuh"]


def _newer(src, dst):
    return not os.path.exists(dst) or os.path.getmtime(src) > os.path.getmtime(dst)


def build(force=False, verbose=False):
    os.makedirs(OUT, exist_ok=True)
    hdr_paths = [os.path.join(CSRC, h) for h in HEADERS]
    hdr_paths.append(os.path.join(os.path.dirname(PKG), "include", "fsgc.h"))
    objs, cmds = [], []
    for s, o, extra in SOURCES:
        src = os.path.join(CSRC, s)
        obj = os.path.join(OUT, o)
        objs.append(obj)
        stale = force or _newer(src, obj) or any(_newer(h, obj) for h in hdr_paths)
        if not stale:
            continue
        if s.endswith(".cu"):
            cmd = [NVCC] + ARCH + COMMON + extra + ["-c", src, "-o", obj] + (["-Xptxas", "-v"] if verbose else [])
        else:
            cmd = [NVCC, "-x", "cu"] + ARCH + COMMON + extra + ["-c", src, "-o", obj]
        cmds.append(cmd)
    from concurrent.futures import ThreadPoolExecutor

    def run(cmd):
        if verbose:
            print(" ".join(cmd), flush=True)
        return subprocess.run(cmd, capture_output=not verbose, text=True)

    with ThreadPoolExecutor(max_workers=max(1, min(len(cmds), os.cpu_count() or 1))) as ex:
        for cmd, r in zip(cmds, ex.map(run, cmds)):
            if r.returncode != 0:
                sys.stderr.write((r.stderr or "") + (r.stdout or ""))
                raise subprocess.CalledProcessError(r.returncode, cmd)
    if force or any(_newer(o, LIB) for o in objs):
        cmd = [NVCC] + ARCH + ["-shared", "-cudart", "static", "-Xcompiler", "-fPIC", "-o", LIB] + objs
        if verbose:
            print(" ".join(cmd), flush=True)
        subprocess.run(cmd, check=True)
    return LIB


if __name__ == "__main__":
    build(force="--force" in sys.argv, verbose=True)
