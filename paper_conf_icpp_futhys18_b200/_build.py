"""Build libglp.so in-tree with nvcc for sm_100a (no JIT cache: the .so travels with the repo)."""
from __future__ import annotations

import glob
import os
import subprocess

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
LIB = os.path.join(PKG, "libglp.so")
SOURCES = sorted(glob.glob(os.path.join(PKG, "csrc", "*"))) + [os.path.join(ROOT, "include", "glp.h")]
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")

FLAGS = ["-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-lineinfo", "-std=c++17",
         "-Xcompiler", "-fPIC,-O2", "-shared", "-cudart", "static"]


def stale() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    return any(os.path.getmtime(s) > t for s in SOURCES)


DIAG_LIB = os.path.join(PKG, "libglp_diag.so")


def build(force: bool = False, verbose: bool = False, diag: bool = False) -> str:
    """libglp.so (the product), or with diag=True libglp_diag.so: the same sources compiled with
    -DGLP_DIAG, which adds the work-skipping / cycle-counter hooks of tools/stage_probe.py and
    tools/clk_probe.py (GLP_DEBUG_* environment variables; results are wrong in skip modes).  The
    diagnostic library is never loaded unless GLP_LIB points at it."""
    lib = DIAG_LIB if diag else LIB
    if not force and os.path.exists(lib) and not any(
            os.path.getmtime(s) > os.path.getmtime(lib) for s in SOURCES):
        return lib
    tmp = lib + f".tmp{os.getpid()}"
    cmd = [NVCC, *FLAGS, *(["-DGLP_DIAG"] if diag else []), "-o", tmp,
           os.path.join(PKG, "csrc", "glp.cu")]
    if verbose:
        cmd.insert(1, "-Xptxas=-v")
    subprocess.check_call(cmd)
    os.replace(tmp, lib)
    return lib


TRACKER_LIB = os.path.join(PKG, "libglp_tracker.so")
CUDA = os.environ.get("CUDA_HOME", "/usr/local/cuda")


def build_tracker(force: bool = False) -> str:
    """libglp_tracker.so: the CUPTI resource tracker (csrc/tracker.cpp, include/glp_tracker.h),
    host C++ linked against the toolkit's libcupti."""
    src = [os.path.join(PKG, "csrc", "tracker.cpp"), os.path.join(ROOT, "include", "glp_tracker.h")]
    if not force and os.path.exists(TRACKER_LIB) and not any(
            os.path.getmtime(s) > os.path.getmtime(TRACKER_LIB) for s in src):
        return TRACKER_LIB
    tmp = TRACKER_LIB + f".tmp{os.getpid()}"
    lib64 = os.path.join(CUDA, "lib64")
    subprocess.check_call(["g++", "-O2", "-std=c++17", "-fPIC", "-shared", "-I", os.path.join(CUDA, "include"),
                           "-o", tmp, src[0], "-L", lib64, "-lcupti", f"-Wl,-rpath,{lib64}"])
    os.replace(tmp, TRACKER_LIB)
    return TRACKER_LIB


if __name__ == "__main__":
    import sys
    print(build(force=True, verbose=True, diag="--diag" in sys.argv))
