"""Build libsr.so in-tree: nvcc for the sm_100a kernels, g++ for the host C++, one shared
library with a static CUDA runtime.  Used by __graft_entry__.build() and `python -m
paper_conf_ppopp_jiangha20_b200._build`."""
from __future__ import annotations

import concurrent.futures as cf
import os
import shutil
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
OUT = os.path.join(PKG, "libsr.so")
BUILD = os.path.join(PKG, "build")
CUDA = os.environ.get("CUDA_HOME", "/usr/local/cuda")
NVCC = os.path.join(CUDA, "bin", "nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]

CU = ["exec.cu", "lsh.cu"]
CPP = ["api.cpp", "cluster.cpp", "tiler.cpp"]
HDRS = [os.path.join(CSRC, "internal.h"), os.path.join(ROOT, "include", "sr.h")]


def _stale(obj: str, src: str) -> bool:
    if not os.path.exists(obj):
        return True
    t = os.path.getmtime(obj)
    return any(os.path.getmtime(p) > t for p in [src] + HDRS)


def _compile(src: str, verbose: bool) -> str:
    s = os.path.join(CSRC, src)
    o = os.path.join(BUILD, src + ".o")
    if not _stale(o, s):
        return o
    if src.endswith(".cu"):
        # SR_NVCC_DEFS: extra -D flags for measurement builds (compile-time knobs in exec.cu)
        defs = os.environ.get("SR_NVCC_DEFS", "").split()
        cmd = [NVCC, *ARCH, *defs, "-O3", "-lineinfo", "-std=c++17", "-Xptxas", "-v" if verbose else "-O3",
               "-Xcompiler", "-fPIC,-fopenmp,-O3", "-I", os.path.join(ROOT, "include"), "-c", s, "-o", o]
    else:
        cmd = ["g++", "-O3", "-std=c++17", "-fPIC", "-fopenmp", "-I", os.path.join(CUDA, "include"),
               "-I", os.path.join(ROOT, "include"), "-c", s, "-o", o]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError(f"compile failed: {' '.join(cmd)}\n{r.stdout}\n{r.stderr}")
    if verbose and r.stderr:
        with open(o + ".log", "w") as f:
            f.write(r.stderr)
    return o


def build(verbose: bool = False, force: bool = False) -> str:
    # objects built with other SR_NVCC_DEFS (a measurement build) are never reused
    stamp = os.path.join(BUILD, "nvcc_defs.txt")
    defs = os.environ.get("SR_NVCC_DEFS", "")
    if os.path.isdir(BUILD) and (not os.path.exists(stamp) or open(stamp).read() != defs):
        force = True
    if force and os.path.isdir(BUILD):
        shutil.rmtree(BUILD)
    os.makedirs(BUILD, exist_ok=True)
    with open(stamp, "w") as f:
        f.write(defs)
    with cf.ThreadPoolExecutor(max_workers=min(8, os.cpu_count() or 2)) as ex:
        objs = list(ex.map(lambda s: _compile(s, verbose), CU + CPP))
    if os.path.exists(OUT) and all(os.path.getmtime(OUT) >= os.path.getmtime(o) for o in objs):
        return OUT
    tmp = OUT + ".tmp"
    cmd = [NVCC, *ARCH, "-shared", "--cudart=static", "-o", tmp, *objs, "-Xcompiler", "-fopenmp", "-lgomp"]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError(f"link failed: {' '.join(cmd)}\n{r.stdout}\n{r.stderr}")
    os.replace(tmp, OUT)
    return OUT


if __name__ == "__main__":
    print(build(verbose="-v" in sys.argv, force="-f" in sys.argv))
