#!/usr/bin/env python
"""Bounds-checked build of the SpMV kernels over small matrices (development
tool; compute-sanitizer is closed on the GPU pool).

    python scripts/checked_small.py

Builds libtilespmv.so with -DTSP_CHECKED into /tmp: every blob copy is
checked against the blob array and the kernel's slot, every remainder x read
against n (or the x cache's size), every staged x segment against n, every y
row against m, and every unit / item index against the schedule's sizes; a
failed check is a device assert (the launch fails, this script exits 1).
Then runs every small config, special shape and mode on all three kernels
and compares y with the oracle.  Not part of the product path."""
import os
import subprocess
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    import torch
    from oracle import oracle as O
    from paper_conf_ipps_niuldj0t21_b200 import _build, tilespmv as T
    from synthetic import gen
    lib = "/tmp/libtilespmv_checked.so"
    subprocess.check_call([_build.NVCC] + _build.FLAGS + ["-DTSP_CHECKED", "-o", lib] + _build.SOURCES)
    _build.LIB = lib
    T._lib = None
    T.load(build_if_missing=False)
    mats = [gen.make(n)[0] for n in ("lap2d_37x29", "mixed_small", "rmat12", "stencil27_21", "fem_small")]
    mats += [gen.random_sparse(17, 33, 0.3, seed=1), gen.random_sparse(1, 1, 1.0),
             gen.random_sparse(100, 1, 0.5, seed=2), gen.random_sparse(1, 100, 0.5, seed=3),
             gen.random_sparse(70, 70, 0.95, seed=4, empty_rows=range(16, 32)),
             gen.csr_from_coo(400, 1800, [3] * 900 + list(range(0, 400)),
                              list(range(0, 1800, 2)) + [(7 * i) % 1700 for i in range(400)], seed=17,
                              name="heavy_row")]
    bad = 0
    for A in mats:
        x = gen.dense_x(A.n, 101)
        yref, absy = O.spmv(A, x)
        for mode in ("ADPT", "DEFERRED", "FORCE_CSR", "BYTES"):
            for kernel in ("SM_QUEUE", "DENSE_ROWS", "GATHER"):
                M = T.TiledMatrix.from_host_csr(A, mode=mode, kernel=kernel)
                xd = torch.from_numpy(x).cuda()
                for _ in range(3):  # repeated launches: split-row counters and the x cache refill
                    y = M.run(xd).cpu().numpy()
                torch.cuda.synchronize()
                ok = bool(np.all(np.abs(y - yref) <= 1e-12 * absy + 1e-300))
                bad += not ok
                print(f"{A.name:14s} {mode:9s} {kernel:10s} {'ok' if ok else 'MISMATCH'}", flush=True)
                M.close()
    print("checked_small done, mismatches:", bad, "(a failed bounds check aborts with a device assert)")
    sys.exit(1 if bad else 0)


if __name__ == "__main__":
    main()
