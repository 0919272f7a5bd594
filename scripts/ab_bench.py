#!/usr/bin/env python
"""A/B timing of SpMV kernel variants on one box (development tool).

    python scripts/ab_bench.py WORKLOAD KERNEL[,KERNEL...] [--rounds R] [--steps K]

KERNEL: SM_QUEUE, DENSE_ROWS or AUTO (tilespmv_opts_t.kernel).  Builds one
handle per kernel on enough replicas of the matrix to defeat L2, then times K
back-to-back SpMVs per kernel, interleaving the kernels round by round.  Prints per-variant
median / min microseconds and the HBM fraction.  Not a bench line.
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("workload")
    ap.add_argument("variants")
    ap.add_argument("--rounds", type=int, default=7)
    ap.add_argument("--steps", type=int, default=100)
    ap.add_argument("--mode", default="DEFERRED")
    a = ap.parse_args()
    import numpy as np
    import torch
    from paper_conf_ipps_niuldj0t21_b200 import tilespmv as T
    from synthetic import gen
    peaks = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    peak = float(peaks.get("hbm_copy_gbs") or peaks.get("hbm_gbs") or 6546.6)
    dev = torch.device("cuda", 0)
    A, x = gen.make(a.workload)
    l2 = torch.cuda.get_device_properties(0).L2_cache_size
    hs = {}
    for v in a.variants.split(","):
        kv = int(v) if v.isdigit() else v
        M0 = T.TiledMatrix.from_host_csr(A, mode=a.mode, device=dev, kernel=kv)
        alg = M0.info()["alg_bytes"]
        reps = max(1, int(np.ceil(4 * l2 / max(alg, 1))))
        Ms = [M0] + [T.TiledMatrix.from_host_csr(A, mode=a.mode, device=dev, kernel=kv) for _ in range(reps - 1)]
        xs = [torch.from_numpy(x).to(dev) for _ in range(reps)]
        ys = [torch.empty(A.m, dtype=torch.float64, device=dev) for _ in range(reps)]
        hs[v] = (Ms, xs, ys, alg, M0.kernel_name())
    res = {v: [] for v in hs}
    graphs = {}
    for v, (Ms, xs, ys, alg, name) in hs.items():  # K launches per variant, one graph each
        R = len(Ms)
        for i in range(10):
            Ms[i % R].run(xs[i % R], ys[i % R])
        torch.cuda.synchronize()
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g):
            for i in range(a.steps):
                Ms[i % R].run(xs[i % R], ys[i % R])
        g.replay()
        graphs[v] = g
    torch.cuda.synchronize()
    s = torch.cuda.current_stream()
    for rnd in range(a.rounds):
        for v in hs:
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            torch.cuda.synchronize()
            e0.record(s)
            graphs[v].replay()
            e1.record(s)
            torch.cuda.synchronize()
            res[v].append(e0.elapsed_time(e1) * 1e3 / a.steps)
    for v, (Ms, xs, ys, alg, name) in hs.items():
        t = np.array(res[v])
        print(f"{a.workload} {v:>10} {name:34s} median {np.median(t):9.2f} us  min {t.min():9.2f} us  "
              f"frac(median) {alg / (np.median(t) * 1e-6) / 1e9 / peak:.3f}  reps {len(Ms)}", flush=True)


if __name__ == "__main__":
    main()
