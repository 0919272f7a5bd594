#!/usr/bin/env python
"""Per-item timeline of the warp kernel (development tool).

    python scripts/trace_items.py WORKLOAD [--mode M]

Builds a trace variant of the library (-DTSP_TRACE) under /tmp, runs a few
SpMVs, and prints where a warp's time goes: blob wait (issue -> landed),
compute (landed -> end), items per warp, and the spread of warp finish
times.  Not part of the product path."""
import argparse
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("workload")
    ap.add_argument("--mode", default="DEFERRED")
    a = ap.parse_args()
    import numpy as np
    import torch
    from paper_conf_ipps_niuldj0t21_b200 import _build, tilespmv as T
    lib = "/tmp/libtilespmv_trace.so"
    subprocess.check_call([_build.NVCC] + _build.FLAGS + ["-DTSP_TRACE", "-o", lib] + _build.SOURCES)
    _build.LIB = lib
    L = T.load(build_if_missing=False)
    from synthetic import gen
    A, x = gen.make(a.workload)
    dev = torch.device("cuda", 0)
    M = T.TiledMatrix.from_host_csr(A, mode=a.mode, device=dev)
    g, b, _ = M.launch_shape()
    W = g * (b // 32)
    KT = 192
    buf = torch.zeros(W * KT * 4 + W, dtype=torch.int64, device=dev)
    xd = torch.from_numpy(x).to(dev)
    y = torch.empty(A.m, dtype=torch.float64, device=dev)
    for _ in range(3):
        M.run(xd, y)
    torch.cuda.synchronize()
    import ctypes
    L.tilespmv_debug_set_trace.argtypes = [ctypes.c_void_p]
    L.tilespmv_debug_set_trace(buf.data_ptr())
    M.run(xd, y)
    torch.cuda.synchronize()
    L.tilespmv_debug_set_trace(None)
    hb = buf.cpu().numpy()
    smid = hb[W * KT * 4:]
    t = hb[:W * KT * 4].reshape(W, KT, 4).astype(np.float64)
    valid = t[:, :, 0] > 0
    t0 = t[:, :, 0][valid].min()
    start = np.where(valid, t[:, :, 0] - t0, np.nan)
    landed = np.where(valid, t[:, :, 1] - t0, np.nan)
    end = np.where(valid, t[:, :, 3] - t0, np.nan)
    wait = landed - start
    comp = end - landed
    nitems = valid.sum(1)
    fin = np.nanmax(end, axis=1)
    print(f"{a.workload}: warps {W}, items traced {int(valid.sum())} (first {KT} per warp), "
          f"items/warp mean {nitems.mean():.1f} max {nitems.max()}")
    print(f"kernel span (first stamp -> last end) {np.nanmax(fin) / 1e3:.1f} us")
    for name, v in (("blob wait", wait), ("compute", comp), ("item total", end - start)):
        f = v[valid]
        print(f"{name:11s} us: mean {f.mean() / 1e3:.2f}  p50 {np.percentile(f, 50) / 1e3:.2f}  "
              f"p90 {np.percentile(f, 90) / 1e3:.2f}  p99 {np.percentile(f, 99) / 1e3:.2f}  max {f.max() / 1e3:.2f}")
    print("warp finish us percentiles (10,50,90,99,max):",
          [round(float(np.percentile(fin, q)) / 1e3, 1) for q in (10, 50, 90, 99)], round(float(fin.max()) / 1e3, 1))
    first = start[:, 0]
    print("warp first-item start us (p50, p99, max):", round(float(np.nanpercentile(first, 50)) / 1e3, 2),
          round(float(np.nanpercentile(first, 99)) / 1e3, 2), round(float(np.nanmax(first)) / 1e3, 2))
    sw = np.nansum(wait, 1)
    sc = np.nansum(comp, 1)
    print(f"per-warp totals us: blob wait mean {sw.mean() / 1e3:.1f}, compute mean {sc.mean() / 1e3:.1f}")
    info = hb[:W * KT * 4].reshape(W, KT, 4)[:, :, 2].astype(np.uint64)
    nbytes = ((info >> np.uint64(16)) & np.uint64(0xFFFF)).astype(np.float64)
    ntr = ((info >> np.uint64(8)) & np.uint64(0xFF)).astype(np.int64)
    ntl = (info & np.uint64(31)).astype(np.int64)
    tot = end - start
    v = valid
    print("item classes (count, mean bytes, mean us, us per KB):")
    for name, sel in (("row-group", v & (ntr > 0)), ("tiles", v & (ntr == 0) & (ntl > 0)),
                      ("remainder-only", v & (ntr == 0) & (ntl == 0))):
        if sel.sum():
            print(f"  {name:15s} {int(sel.sum()):7d} {nbytes[sel].mean():8.0f} B {tot[sel].mean() / 1e3:6.2f} us "
                  f"{(tot[sel].mean() / 1e3) / max(nbytes[sel].mean() / 1024, 1e-9):6.2f}")
    # least-squares time ~ a + b * bytes over all traced items
    X = np.stack([np.ones(v.sum()), nbytes[v]], 1)
    coef, *_ = np.linalg.lstsq(X, tot[v], rcond=None)
    print(f"fit: item us ~ {coef[0] / 1e3:.2f} + {coef[1]:.3f} ns/B * bytes  (fixed ~ {coef[0] / max(coef[1], 1e-9):.0f} B)")
    dec = np.array_split(np.arange(W), 10)
    print("mean warp finish by warp-index decile (us):", [round(float(fin[d].mean()) / 1e3, 1) for d in dec])
    sm_fin = np.array([fin[smid == s_].max() if (smid == s_).any() else 0 for s_ in range(int(smid.max()) + 1)])
    sm_mean = np.array([fin[smid == s_].mean() if (smid == s_).any() else 0 for s_ in range(int(smid.max()) + 1)])
    print("per-SM mean warp finish us: min %.1f p50 %.1f max %.1f; SMs with the 5 latest means:" %
          (sm_mean.min() / 1e3, np.median(sm_mean) / 1e3, sm_mean.max() / 1e3), list(np.argsort(sm_mean)[-5:]))
    print("per-SM mean finish by SM id decile:", [round(float(sm_mean[d].mean()) / 1e3, 1)
                                                  for d in np.array_split(np.arange(sm_mean.size), 10)])
    slow = np.argsort(fin)[-5:]
    for w in slow:
        print(f"  slow warp {w}: items {nitems[w]}, finish {fin[w] / 1e3:.1f} us, wait {sw[w] / 1e3:.1f}, "
              f"compute {sc[w] / 1e3:.1f}")


if __name__ == "__main__":
    main()
