#!/usr/bin/env python
"""Interleaved A/B of several builds of libtilespmv.so in ONE process
(development tool, not a bench line).

    python scripts/ab_libs.py WL[:MODE],... LIB1.so,LIB2.so,... [--rounds R] [--steps K]

Each matrix is generated once; every library gets its own handles on enough
replicas to defeat L2, K back-to-back launches captured in one CUDA graph,
and the graphs replay round-robin R times.  Prints per library: median/min
us per SpMV, the HBM fraction, a single-launch median (one launch between two
events with the stream held by a spin kernel), whether y equals the first
library's bitwise, and the largest |y - y_first| / (|A||x|).
"""
import argparse
import ctypes
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("workloads")
    ap.add_argument("libs")
    ap.add_argument("--rounds", type=int, default=5)
    ap.add_argument("--steps", type=int, default=100)
    ap.add_argument("--single", type=int, default=30)
    a = ap.parse_args()
    import numpy as np
    import scipy.sparse as sp
    import torch
    from paper_conf_ipps_niuldj0t21_b200 import tilespmv as T
    from synthetic import gen
    peaks = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    peak = float(peaks.get("hbm_copy_gbs") or peaks.get("hbm_gbs") or 6546.6)
    dev = torch.device("cuda", 0)
    l2 = torch.cuda.get_device_properties(0).L2_cache_size
    libs = a.libs.split(",")
    loaded = {}
    for path in libs:
        T._lib = None
        T._build.LIB = os.path.abspath(path)
        loaded[path] = T.load(build_if_missing=False)
    spin = torch.empty(1, device=dev)
    for wlm in a.workloads.split(","):
        wl, mode = (wlm.split(":") + ["DEFERRED"])[:2]
        A, x = gen.make(wl)
        S = sp.csr_matrix((np.abs(A.val), A.colidx, A.rowptr), shape=(A.m, A.n))
        absy = S @ np.abs(x)
        hs = {}
        for path in libs:
            T._lib = loaded[path]
            M0 = T.TiledMatrix.from_host_csr(A, mode=mode, device=dev)
            alg = M0.info()["alg_bytes"]
            reps = max(1, int(np.ceil(4 * l2 / max(alg, 1))))
            Ms = [M0] + [T.TiledMatrix.from_host_csr(A, mode=mode, device=dev) for _ in range(reps - 1)]
            xs = [torch.from_numpy(x).to(dev) for _ in range(reps)]
            ys = [torch.empty(A.m, dtype=torch.float64, device=dev) for _ in range(reps)]
            R = len(Ms)
            for i in range(10):
                Ms[i % R].run(xs[i % R], ys[i % R])
            torch.cuda.synchronize()
            y = ys[0].cpu().numpy().copy()
            g = torch.cuda.CUDAGraph()
            with torch.cuda.graph(g):
                for i in range(a.steps):
                    Ms[i % R].run(xs[i % R], ys[i % R])
            g.replay()
            torch.cuda.synchronize()
            hs[path] = dict(Ms=Ms, xs=xs, ys=ys, alg=alg, g=g, y=y, name=M0.kernel_name(), t=[], s=[])
        s = torch.cuda.current_stream()
        for rnd in range(a.rounds):
            for path, h in hs.items():
                T._lib = loaded[path]
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                torch.cuda.synchronize()
                e0.record(s)
                h["g"].replay()
                e1.record(s)
                torch.cuda.synchronize()
                h["t"].append(e0.elapsed_time(e1) * 1e3 / a.steps)
        for rnd in range(a.single):
            for path, h in hs.items():
                T._lib = loaded[path]
                R = len(h["Ms"])
                i = rnd % R
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                torch.cuda.synchronize()
                torch.cuda._sleep(200000)
                e0.record(s)
                h["Ms"][i].run(h["xs"][i], h["ys"][i])
                e1.record(s)
                torch.cuda.synchronize()
                h["s"].append(e0.elapsed_time(e1) * 1e3)
        y0 = hs[libs[0]]["y"]
        for path, h in hs.items():
            t = np.array(h["t"])
            same = bool(np.array_equal(h["y"].view(np.uint64), y0.view(np.uint64)))
            rel = float(np.max(np.abs(h["y"] - y0) / (absy + 1e-300)))
            print(f"{wl:>14s}:{mode:<8s} {os.path.basename(path):>14s} {h['name']:28s} median {np.median(t):8.2f} us"
                  f"  min {t.min():8.2f}  frac {h['alg'] / (np.median(t) * 1e-6) / 1e9 / peak:.3f}"
                  f"  single {np.median(h['s']):7.2f} us  bitwise {same}  maxrel {rel:.1e}", flush=True)
        for path, h in hs.items():  # each handle destroyed by its own library
            T._lib = loaded[path]
            h["g"] = None
            for M in h["Ms"]:
                M.close()
        del hs
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
