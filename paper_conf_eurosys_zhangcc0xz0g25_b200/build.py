"""Build the native library ``lib/libbless.so`` in-tree (sm_100a).

C++17 host code (scheduler, engine, C ABI) is compiled with g++; CUDA sources
with nvcc ``-gencode arch=compute_100a,code=sm_100a -lineinfo``.  The CUDA
runtime is linked statically so the library does not depend on which
libcudart a host process (e.g. torch) has loaded.  Incremental: an object is
rebuilt when its source or any header under csrc/ or include/ is newer.
"""
from __future__ import annotations

import concurrent.futures as cf
import glob
import os
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
OBJ = os.path.join(PKG, "build_obj")
LIBDIR = os.path.join(PKG, "lib")
LIB = os.path.join(LIBDIR, "libbless.so")
CUDA = os.environ.get("CUDA_HOME", "/usr/local/cuda")
NVCC = os.path.join(CUDA, "bin", "nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
INC = ["-I" + os.path.join(ROOT, "include"), "-I" + os.path.join(CUDA, "include")]
CXXFLAGS = ["-std=c++17", "-O2", "-fPIC", "-Wall", "-Wno-unused-function"]
NVFLAGS = ["-std=c++17", "-O3", "-lineinfo", "--expt-relaxed-constexpr", "-Xcompiler", "-fPIC",
           "-Xptxas", "-v"] + ARCH


def _sources():
    cpp = sorted(glob.glob(os.path.join(CSRC, "**", "*.cpp"), recursive=True))
    cu = sorted(glob.glob(os.path.join(CSRC, "**", "*.cu"), recursive=True))
    return cpp, cu


def _headers_mtime():
    hs = glob.glob(os.path.join(CSRC, "**", "*.h*"), recursive=True) + \
        glob.glob(os.path.join(CSRC, "**", "*.cuh"), recursive=True) + \
        glob.glob(os.path.join(ROOT, "include", "**", "*.h"), recursive=True)
    return max((os.path.getmtime(h) for h in hs), default=0.0)


def _obj_path(src):
    rel = os.path.relpath(src, CSRC).replace(os.sep, "__")
    return os.path.join(OBJ, rel + ".o")


def _compile(src, verbose):
    out = _obj_path(src)
    if src.endswith(".cu"):
        extra = os.environ.get("BLESS_EXTRA_NVFLAGS", "").split()   # debug builds (e.g. -DBLESS_TC_TRACE)
        cmd = [NVCC] + NVFLAGS + extra + INC + ["-c", src, "-o", out]
    else:
        cmd = ["g++"] + CXXFLAGS + INC + ["-c", src, "-o", out]
    r = subprocess.run(cmd, capture_output=True, text=True)
    log = r.stdout + r.stderr
    if r.returncode != 0:
        raise RuntimeError(f"compile failed: {' '.join(cmd)}\n{log}")
    if verbose and log.strip():
        with open(out + ".log", "w") as f:
            f.write(log)
    return out


def build(force: bool = False, verbose: bool = True, jobs: int | None = None) -> str:
    os.makedirs(OBJ, exist_ok=True)
    os.makedirs(LIBDIR, exist_ok=True)
    cpp, cu = _sources()
    hdr = _headers_mtime()
    todo = []
    for s in cpp + cu:
        o = _obj_path(s)
        if force or not os.path.exists(o) or os.path.getmtime(o) < max(os.path.getmtime(s), hdr):
            todo.append(s)
    if todo:
        with cf.ThreadPoolExecutor(max_workers=jobs or min(8, os.cpu_count() or 4)) as ex:
            list(ex.map(lambda s: _compile(s, verbose), todo))
    objs = [_obj_path(s) for s in cpp + cu]
    if todo or not os.path.exists(LIB) or os.path.getmtime(LIB) < max(os.path.getmtime(o) for o in objs):
        cmd = ["g++", "-shared", "-o", LIB] + objs + [
            "-L" + os.path.join(CUDA, "lib64"), "-lcudart_static", "-lpthread", "-ldl", "-lrt"]
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode != 0:
            raise RuntimeError(f"link failed: {' '.join(cmd)}\n{r.stdout}{r.stderr}")
    return LIB


if __name__ == "__main__":
    print(build(force="--force" in sys.argv))
