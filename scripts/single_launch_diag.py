#!/usr/bin/env python
"""Where does a single SpMV launch's time go?  (development tool)

    python scripts/single_launch_diag.py WORKLOAD [MODE]

Times one launch between two events in several settings (median of 40):
  held     stream held by a spin kernel while event/launch/event are enqueued
  warm     as held, but a launch of another replica precedes the first event
           (the SM shared-memory carve-out is already the kernel's)
  idle     stream idle, events recorded around a launch from Python
  graph    as held, the launch replayed from a one-node CUDA graph
and, for scale, the same settings for a 1-element torch kernel (the launch
floor) and a torch copy moving the SpMV's algorithmic bytes (half read, half
written; replicas rotated so L2 holds none of it).
"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_niuldj0t21_b200 import TiledMatrix  # noqa: E402
from synthetic import gen  # noqa: E402

wl = sys.argv[1]
mode = sys.argv[2] if len(sys.argv) > 2 else "DEFERRED"
dev = torch.device("cuda", 0)
A, x = gen.make(wl)
R = 8
Ms = [TiledMatrix.from_host_csr(A, mode=mode, device=dev) for _ in range(R)]
xs = [torch.from_numpy(x).to(dev) for _ in range(R)]
ys = [torch.empty(A.m, dtype=torch.float64, device=dev) for _ in range(R)]
s = torch.cuda.current_stream()
g = torch.cuda.CUDAGraph()
with torch.cuda.graph(g):
    Ms[0].run(xs[0], ys[0])
torch.cuda.synchronize()


tiny = torch.zeros(1, device=dev)
alg0 = Ms[0].info()["alg_bytes"]
half = alg0 // 16  # doubles per copy side
srcs = [torch.rand(half, dtype=torch.float64, device=dev) for _ in range(R)]
dsts = [torch.empty_like(srcs[0]) for _ in range(R)]


def t(kind, n=40, what="spmv"):
    out = []
    for i in range(n + 3):
        j = i % R
        if what != "spmv":
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            torch.cuda.synchronize()
            torch.cuda._sleep(400_000)
            e0.record(s)
            if what == "tiny":
                tiny.add_(1.0)
            else:
                dsts[j].copy_(srcs[j])
            e1.record(s)
            torch.cuda.synchronize()
            if i >= 3:
                out.append(e0.elapsed_time(e1) * 1e3)
            continue
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        if kind != "idle":
            torch.cuda._sleep(400_000)
        if kind == "warm":
            Ms[(j + 1) % R].run(xs[(j + 1) % R], ys[(j + 1) % R])
        e0.record(s)
        if kind == "graph":
            g.replay()
        else:
            Ms[j].run(xs[j], ys[j])
        e1.record(s)
        torch.cuda.synchronize()
        if i >= 3:
            out.append(e0.elapsed_time(e1) * 1e3)
    return np.median(out)


alg = Ms[0].info()["alg_bytes"]
for kind in ("held", "warm", "idle", "graph", "held", "warm"):
    us = t(kind)
    print(f"{wl}/{mode} {kind:6s} {us:8.2f} us  frac {alg / (us * 1e-6) / 1e9 / 6547.8:.3f}", flush=True)
for what in ("tiny", "copy", "tiny", "copy"):
    us = t("held", what=what)
    print(f"{what:5s} (held) {us:8.2f} us" + (f"  copy of {alg0 / 1e6:.1f} MB traffic: frac {alg0 / (us * 1e-6) / 1e9 / 6547.8:.3f}" if what == "copy" else ""), flush=True)
