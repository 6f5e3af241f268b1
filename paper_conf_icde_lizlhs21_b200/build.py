"""Builds libdyc.so in-tree with nvcc for sm_100a (no torch extension machinery).

    python -m paper_conf_icde_lizlhs21_b200.build
"""
from __future__ import annotations

import os
import shutil
import subprocess

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
INCLUDE = os.path.join(ROOT, "include")
LIB = os.path.join(PKG, "libdyc.so")
SOURCES = ["dyc_api.cu", "dyc_dist.cu"]
DEPS = SOURCES + ["dyc_kernels.cuh", "dyc_device.cuh", "dyw_api.cuh", "dyw_kernels.cuh"]

COMPILE_FLAGS = [
    "-O3", "-std=c++17", "-lineinfo",
    "-gencode", "arch=compute_100a,code=sm_100a",
    "-Xcompiler", "-fPIC,-O2",
]
LINK_FLAGS = ["-shared", "-cudart", "static", "-gencode", "arch=compute_100a,code=sm_100a", "-ldl"]
NVCC_FLAGS = COMPILE_FLAGS + LINK_FLAGS


def nvcc_path() -> str:
    for cand in (shutil.which("nvcc"), "/usr/local/cuda/bin/nvcc"):
        if cand and os.path.exists(cand):
            return cand
    raise RuntimeError("nvcc not found: cannot build libdyc.so")


def needs_build() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    files = [os.path.join(CSRC, f) for f in DEPS] + [os.path.join(INCLUDE, h) for h in ("dycuckoo.h", "dycuckoo_wide.h")]
    return any(os.path.getmtime(f) > t for f in files)


def build_library(force: bool = False, verbose: bool = False) -> str:
    """Compiles every source to an object in parallel (nvcc -c), then links
    libdyc.so (static cudart, -ldl for the run-time NCCL load of dyc_dist.cu)."""
    if not force and not needs_build():
        return LIB
    tag = f".tmp{os.getpid()}"
    objs, procs = [], []
    for src in SOURCES:
        obj = os.path.join(PKG, src.replace(".cu", tag + ".o"))
        cmd = [nvcc_path(), *COMPILE_FLAGS, "-I", INCLUDE, "-c", "-o", obj, os.path.join(CSRC, src)]
        if verbose:
            print(" ".join(cmd))
        procs.append(subprocess.Popen(cmd))
        objs.append(obj)
    rcs = [p.wait() for p in procs]
    try:
        if any(rcs):
            raise subprocess.CalledProcessError(max(rcs), "nvcc -c")
        tmp = LIB + tag
        cmd = [nvcc_path(), *LINK_FLAGS, "-o", tmp] + objs
        if verbose:
            print(" ".join(cmd))
        subprocess.check_call(cmd)
        os.replace(tmp, LIB)
    finally:
        for o in objs:
            if os.path.exists(o):
                os.remove(o)
    return LIB


if __name__ == "__main__":
    print(build_library(force=True, verbose=True))
