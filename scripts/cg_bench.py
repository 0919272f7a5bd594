#!/usr/bin/env python
"""CG on the tiled SpMV, measured (development /
reporting tool, not the bench line).

    python scripts/cg_bench.py [--workload stencil27_200] [--iters 100]

A is the 27-point stencil with its closed-form values (26 on the diagonal,
-1 off it: symmetric positive definite with the Dirichlet boundary), b = A.1.
tilespmv_cg runs `iters` iterations with tol = 0 (so none stops early); the
time per iteration is set beside one tiled SpMV and the iteration's bytes:
the SpMV's algorithmic bytes plus 88 B per row for the three fused vector
kernels (p.q: read p, q; update: read x, r, p, q, write x, r; direction:
read r, p, write p).  One JSON line.
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--workload", default="stencil27_200")
    ap.add_argument("--iters", type=int, default=100)
    a = ap.parse_args()
    import numpy as np
    import torch
    from paper_conf_ipps_niuldj0t21_b200 import TiledMatrix
    from synthetic import gen
    nx = int(a.workload.rsplit("_", 1)[1])
    A = gen.stencil27(nx, values="stencil")
    dev = torch.device("cuda", 0)
    M = TiledMatrix.from_host_csr(A, mode="DEFERRED", device=dev)
    info = M.info()
    ones = torch.ones(A.n, dtype=torch.float64, device=dev)
    b = M.run(ones)
    # warm-up: a short solve and a few SpMVs
    M.cg(b, tol=0.0, maxit=5)
    y = torch.empty(A.m, dtype=torch.float64, device=dev)
    for _ in range(5):
        M.run(ones, y)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(50):
        M.run(ones, y)
    e1.record()
    torch.cuda.synchronize()
    spmv_ms = e0.elapsed_time(e1) / 50
    e0.record()
    x, it, rel = M.cg(b, tol=0.0, maxit=a.iters)
    e1.record()
    torch.cuda.synchronize()
    cg_ms = e0.elapsed_time(e1)
    # the solution of A x = A 1 is 1: report how close the solve got
    err = float((x - 1.0).abs().max())
    peaks = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json"))) if os.path.exists(
        os.path.join(ROOT, "MEASURED_PEAKS.json")) else {}
    peak = float(peaks.get("hbm_gbs") or 6546.6)
    it_ms = cg_ms / max(it, 1)
    it_bytes = info["alg_bytes"] + 88 * A.m
    print(json.dumps({
        "workload": a.workload, "values": "stencil (26 / -1), b = A.1", "n": A.n, "nnz": A.nnz,
        "iterations": it, "relres": rel, "max_abs_err_vs_ones": err,
        "cg_ms_per_iter": it_ms, "spmv_ms": spmv_ms, "spmv_share_of_iter": spmv_ms / it_ms,
        "iter_bytes": it_bytes, "iter_gbs": it_bytes / it_ms / 1e6, "hbm_peak_gbs": peak,
        "iter_frac_of_peak": it_bytes / it_ms / 1e6 / peak,
        "kernel": M.kernel_name()}))


if __name__ == "__main__":
    main()
