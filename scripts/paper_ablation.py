#!/usr/bin/env python
"""Paper-figure analogues on B200 (SURVEY §8(f) f2 + f3), one JSON line per
(workload, mode):

  * Fig. 6: TileSpMV_CSR (FORCE_CSR) vs TileSpMV_ADPT vs
    TileSpMV_DeferredCOO (and AUTO, the 1.8M switch of P:235, reading R18)
    GFLOP/s of the same matrix, plus the optional byte-cost selection
    (BYTES; not the paper's rule);
  * Fig. 7: tiles and nonzeros per format (ADPT selection);
  * Fig. 10: space of the tiled form against plain CSR
    (12 B per nonzero + 4 B per row pointer);
  * Fig. 11: preprocessing time (the GPU tiler, create) against
    one SpMV.

    python scripts/paper_ablation.py [--workloads a,b,...] [--modes ...] [--steps K]

Timing as bench.py: K back-to-back launches replayed from one CUDA graph,
rotating replicas when the working set is under 4x L2.  Development /
reporting tool, not the bench line.
"""
import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

FMTS = ["CSR", "COO", "ELL", "HYB", "DNS", "DNSROW", "DNSCOL"]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--workloads", default="lap2d_64,fem,rmat20,mixed,stencil27_200")
    ap.add_argument("--modes", default="FORCE_CSR,ADPT,DEFERRED,AUTO,BYTES")
    ap.add_argument("--steps", type=int, default=100)
    a = ap.parse_args()
    import numpy as np
    import torch
    from paper_conf_ipps_niuldj0t21_b200 import TiledMatrix
    from synthetic import gen
    peak = float(json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"])
    dev = torch.device("cuda", 0)
    L2 = torch.cuda.get_device_properties(0).L2_cache_size
    s = torch.cuda.current_stream()
    for wl in a.workloads.split(","):
        A, x = gen.make(wl)
        rp = torch.from_numpy(A.rowptr).to(dev)
        ci = torch.from_numpy(A.colidx).to(dev)
        va = torch.from_numpy(A.val).to(dev)
        csr_bytes = 12 * A.nnz + 4 * (A.m + 1)
        for mode in a.modes.split(","):
            torch.cuda.synchronize()
            t = time.perf_counter()
            M0 = TiledMatrix.from_csr(rp, ci, va, A.m, A.n, mode=mode)
            create_ms = (time.perf_counter() - t) * 1e3
            info = M0.info()
            reps = max(1, -(-4 * L2 // max(info["alg_bytes"], 1)))
            Ms = [M0] + [TiledMatrix.from_csr(rp, ci, va, A.m, A.n, mode=mode) for _ in range(reps - 1)]
            xs = [torch.from_numpy(x).to(dev) for _ in range(reps)]
            ys = [torch.empty(A.m, dtype=torch.float64, device=dev) for _ in range(reps)]
            for i in range(5):
                Ms[i % reps].run(xs[i % reps], ys[i % reps])
            torch.cuda.synchronize()
            g = torch.cuda.CUDAGraph()
            with torch.cuda.graph(g):
                for i in range(a.steps):
                    Ms[i % reps].run(xs[i % reps], ys[i % reps])
            g.replay()
            torch.cuda.synchronize()
            ts = []
            for _ in range(5):
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(s)
                g.replay()
                e1.record(s)
                torch.cuda.synchronize()
                ts.append(e0.elapsed_time(e1) / a.steps)
            ms = float(np.median(ts))
            out = {"workload": wl, "mode": mode, "resolved_mode": info["mode"], "m": A.m, "nnz": A.nnz,
                   "kernel": M0.kernel_name(), "spmv_us": ms * 1e3,
                   "gflops": 2.0 * A.nnz / (ms * 1e-3) / 1e9,
                   "alg_gbs": info["alg_bytes"] / (ms * 1e-3) / 1e9,
                   "frac_of_peak": info["alg_bytes"] / (ms * 1e-3) / 1e9 / peak,
                   "replicas": reps,
                   # Fig. 7: format mix chosen by the ADPT rules, and kept after extraction
                   "sel_tiles": dict(zip(FMTS, info["sel_tiles"])), "sel_nnz": dict(zip(FMTS, info["sel_nnz"])),
                   "kept_tiles": dict(zip(FMTS, info["kept_tiles"])), "rem_nnz": info["rem_nnz"],
                   # Fig. 10: space
                   "csr_bytes": csr_bytes, "payload_bytes": info["payload_bytes"],
                   "meta_bytes": info["meta_bytes"], "alg_bytes": info["alg_bytes"],
                   "tiled_over_csr": (info["payload_bytes"] + info["meta_bytes"] + 12 * info["rem_nnz"]
                                      + (4 * (A.m + 1) if info["rem_nnz"] else 0)) / csr_bytes,
                   "device_bytes": info["device_bytes"],
                   # Fig. 11: preprocessing against one SpMV
                   "create_ms": create_ms, "create_over_spmv": create_ms / ms}
            print(json.dumps(out), flush=True)
            for M in Ms:
                M.close()
            del xs, ys
            torch.cuda.empty_cache()
        del rp, ci, va


if __name__ == "__main__":
    main()
