"""Builds libtilespmv.so in-tree with nvcc for sm_100a (no JIT cache)."""
from __future__ import annotations

import os
import subprocess

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
LIB = os.path.join(PKG, "libtilespmv.so")
SOURCES = [os.path.join(PKG, "csrc", f)
           for f in ("abi.cu", "tiler.cu", "schedule.cu", "spmv_warp.cu", "cg.cu")]
HEADERS = [os.path.join(PKG, "csrc", f) for f in ("internal.cuh", "spmv_common.cuh", "spmv_tiles.cuh")] + \
          [os.path.join(ROOT, "include", "tilespmv.h")]
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
FLAGS = ["-gencode", "arch=compute_100a,code=sm_100a", "-lineinfo", "-O3", "-std=c++17",
         "-Xcompiler", "-fPIC", "-shared", "-t", "3"]


def stale() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    return any(os.path.getmtime(s) > t for s in SOURCES + HEADERS)


def build(force: bool = False, verbose: bool = False) -> str:
    if force or stale():
        cmd = [NVCC] + FLAGS + (["-Xptxas", "-v"] if verbose else []) + ["-o", LIB] + SOURCES
        subprocess.check_call(cmd)
    return LIB
