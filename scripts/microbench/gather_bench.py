#!/usr/bin/env python
"""Runs gather_bench.cu on the R-MAT 2^20 column stream (development tool).
Prints microseconds and effective GB/s (12 B/entry + 8 B/gather) per variant."""
import ctypes, os, subprocess, sys
import numpy as np
import torch
HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(os.path.dirname(HERE))
sys.path.insert(0, ROOT)
from synthetic import gen  # noqa: E402
so = os.path.join(HERE, "gather_bench.so")
subprocess.check_call(["/usr/local/cuda/bin/nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-shared",
                       "-Xcompiler", "-fPIC", "-o", so, os.path.join(HERE, "gather_bench.cu")])
L = ctypes.CDLL(so)
p = ctypes.c_void_p
L.gather_bench.argtypes = [ctypes.c_int] * 5 + [p, p, p, ctypes.c_int64, p, ctypes.c_int, ctypes.POINTER(ctypes.c_float)]
name = sys.argv[1] if len(sys.argv) > 1 else "rmat20"
A, x = gen.make(name)
dev = torch.device("cuda", 0)
col = torch.from_numpy(A.colidx).to(dev)
val = torch.from_numpy(A.val).to(dev)
xd = torch.from_numpy(x).to(dev)
perm = torch.randperm(A.nnz, device=dev)
colr = col[perm].contiguous()  # same columns, random order
out = torch.empty(148 * 2048, dtype=torch.float64, device=dev)
n = A.nnz
print(f"{name}: {n} entries, x {8 * A.n / 1e6:.1f} MB", flush=True)
sweep = [(148, 1024, k * 1024) for k in (0, 16, 32, 48, 64, 80, 100, 128, 160, 200, 220)]
sweep += [(296, 512, k * 1024) for k in (0, 32, 50, 64, 100)]
for cname, c in (("rowmajor", col),):
    for kind, kn in ((0, "nc"), (3, "ca")):
        for u in (4,):
            for (blocks, threads, smem) in sweep:
                ms = ctypes.c_float()
                rc = L.gather_bench(kind, u, blocks, threads, smem, c.data_ptr(), val.data_ptr(), xd.data_ptr(), n,
                                    out.data_ptr(), 20, ctypes.byref(ms))
                if rc:
                    continue
                us = ms.value * 1e3
                print(f"{cname:9s} {kn:20s} U={u} grid={blocks:4d}x{threads} smem={smem // 1024:3d}K "
                      f"{us:8.1f} us  {n * 20 / (us * 1e-6) / 1e9:7.0f} GB/s  stream-only-frac {n * 12 / (us * 1e-6) / 1e9 / 6547.8:.3f}",
                      flush=True)
