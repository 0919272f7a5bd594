#!/usr/bin/env python
"""gather_bench.cu KIND 5 on the R-MAT stream: the K most-gathered 128-byte
x lines allocate in L1, the others are read with L1::no_allocate (development
tool).  Compared with KIND 0 (all allocate) and KIND 4 (none)."""
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
val = torch.from_numpy(A.val).to(dev)
xd = torch.from_numpy(x).to(dev)
out = torch.empty(148 * 2048, dtype=torch.float64, device=dev)
n = A.nnz
line = A.colidx >> 4
cnt = np.bincount(line)
order = np.argsort(-cnt, kind="stable")
print(f"{name}: {n} entries, x {8 * A.n / 1e6:.1f} MB, {len(cnt)} lines", flush=True)
def run(kind, colv, smem, tag):
    c = torch.from_numpy(colv).to(dev)
    ms = ctypes.c_float()
    rc = L.gather_bench(kind, 4, 148, 1024, smem, c.data_ptr(), val.data_ptr(), xd.data_ptr(), n, out.data_ptr(), 20, ctypes.byref(ms))
    us = ms.value * 1e3
    print(f"{tag:28s} smem={smem // 1024:3d}K rc={rc} {us:8.1f} us  stream-only-frac {n * 12 / (us * 1e-6) / 1e9 / 6547.8:.3f}", flush=True)
for smem in (0, 132 * 1024, 222 * 1024):
    run(0, A.colidx, smem, "all allocate (nc)")
    run(4, A.colidx, smem, "none allocate")
    for K in (128, 256, 512, 768, 1024, 1536, 2048, 4096):
        hot = np.zeros(len(cnt), bool); hot[order[:K]] = True
        cov = cnt[order[:K]].sum() / n
        colv = np.where(hot[line], A.colidx, A.colidx | np.int32(-2**31)).astype(np.int32)
        run(5, colv, smem, f"hot {K} lines ({cov:.2f} of gathers)")
