#!/usr/bin/env python
"""Benchmark of the B200 tiled fp64 SpMV hot path (TileSpMV, IPDPS'21).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]
                    [--workload stencil27_200|fem|rmat20|mixed|lap2d_64] [--mode DEFERRED]

One "step" is one pass of the whole hot path over one batch of synthetic input:
the single-kernel tiled SpMV y = A x (N = 1), or, tile-row sharded over N
GPUs, each rank's SpMV of its tile rows followed by the NCCL all-gather of y
(N > 1).  The matrix is built once (GPU tiler, not timed).  Inputs are resident
in HBM when the timed region starts; working sets smaller than 4x L2 rotate
over independent replicas so every step streams from HBM.

Prints ONE JSON line on rank 0 (the driver contract): metric/value/unit,
roofline of the SpMV kernel against MEASURED_PEAKS.json, the CPU oracle
baseline, an end-to-end number through the host-buffer C-ABI call, clocks.
"""
from __future__ import annotations

import argparse
import json
import os
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "fp64 SpMV GFLOP/s (2*nnz/t)"
UNIT = "GFLOP/s"
DEFAULT_WORKLOAD = "stencil27_200"
WORKLOAD_DESC = {
    "stencil27_200": "3D 27-point stencil 200^3 (8M rows, 213.8M nnz) [BASELINE configs[4]]",
    "fem": "FEM-like banded block matrix, cant-shaped, 62,464 rows, 4.06M nnz [configs[1]]",
    "rmat20": "R-MAT 2^20, edge factor 16, 16.09M nnz [configs[2]]",
    "mixed": "mixed 7-format synthetic, 2^20 rows, 45.6M nnz [configs[3]]",
    "lap2d_64": "2D 5-point Laplacian 64x64 [configs[0]]",
}


def log(*a):
    print(*a, file=sys.stderr, flush=True)


# --------------------------------------------------------------------------
# environment helpers
# --------------------------------------------------------------------------

def hbm_peak():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    try:
        with open(p) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs, copy test)"
    except Exception:
        return 6650.0, "fallback (B200_PROFILING.md)"


def profile_traffic(workload: str, mode: str):
    """dram__bytes_read.sum + dram__bytes_write.sum per launch of the SpMV
    kernel from the committed ncu --set full capture (profiles/)."""
    p = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    try:
        with open(p) as f:
            d = json.load(f)
        return d.get(f"{workload}/{mode}")
    except Exception:
        return None


class ClockSampler:
    """NVML sampling of SM clock and throttle reasons during the timed region."""

    REASONS = {0x1: "gpu_idle", 0x2: "applications_clocks_setting", 0x4: "sw_power_cap",
               0x8: "hw_slowdown", 0x10: "sync_boost", 0x20: "sw_thermal_slowdown",
               0x40: "hw_thermal_slowdown", 0x80: "hw_power_brake_slowdown",
               0x100: "display_clock_setting"}

    def __init__(self, index: int):
        self.samples, self.reasons = [], 0
        self.max_mhz = None
        self._stop = threading.Event()
        self.ok = False
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
            self.ok = True
        except Exception as e:  # pragma: no cover
            log("clock sampler unavailable:", e)

    def _run(self):
        while not self._stop.is_set():
            try:
                t = time.perf_counter()
                mhz = self.nv.nvmlDeviceGetClockInfo(self.h, self.nv.NVML_CLOCK_SM)
                rs = int(self.nv.nvmlDeviceGetCurrentClocksEventReasons(self.h))
                self.samples.append((t, mhz, rs))
            except Exception:
                pass
            time.sleep(0.002)

    def __enter__(self):
        # started before the warm-up so that thread start and NVML set-up never
        # fall inside the timed region; window() marks the timed region
        if self.ok:
            self.t = threading.Thread(target=self._run, daemon=True)
            self.t.start()
            while not self.samples and self.t.is_alive():
                time.sleep(0.001)
        return self

    def __exit__(self, *a):
        self._stop.set()
        if self.ok:
            self.t.join()

    def window(self, t0, t1):
        self.t0, self.t1 = t0, t1

    def summary(self):
        if not self.ok:
            return None
        t0, t1 = getattr(self, "t0", -1e30), getattr(self, "t1", 1e30)
        inside = [s for s in self.samples if t0 <= s[0] <= t1]
        if not inside and self.samples:  # timed region shorter than one sample period
            inside = [min(self.samples, key=lambda s: abs(s[0] - 0.5 * (t0 + t1)))]
        reasons = 0
        for s in inside:
            reasons |= s[2]
        rs = [name for bit, name in self.REASONS.items() if reasons & bit and name != "gpu_idle"]
        return {"sm_mhz": float(np.median([s[1] for s in inside])) if inside else None,
                "sm_max_mhz": self.max_mhz, "samples": len(inside), "reasons": rs}


# --------------------------------------------------------------------------
# workload construction (synthetic, seeded)
# --------------------------------------------------------------------------

def tile_row_bounds(nrows_total: int, P: int, weights=None):
    """Contiguous tile-row ranges, 16-row aligned; balanced by weights (per
    tile row) if given, else by count.  Returns row boundaries [P+1]."""
    from paper_conf_ipps_niuldj0t21_b200.sharded import partition_tile_rows
    return partition_tile_rows(nrows_total, P, weights)


def build_local(workload: str, rank: int, P: int):
    """The rank's row slice of the workload (all rows at P = 1)."""
    from synthetic import gen
    if workload.startswith("stencil27_"):
        nx = int(workload.split("_")[1])
        m = nx ** 3
        b = tile_row_bounds(m, P)
        A = gen.stencil27(nx, row_range=(b[rank], b[rank + 1]))
        A.name = workload
        return A, m, m, b
    A, _ = gen.make(workload)
    w = np.diff(A.rowptr[np.minimum(np.arange(0, A.m + 16, 16), A.m)].astype(np.int64))
    b = tile_row_bounds(A.m, P, w)
    S = A.row_slice(b[rank], b[rank + 1]) if P > 1 else A
    S.name = workload
    return S, A.m, A.n, b


# --------------------------------------------------------------------------
# CPU oracle timing (the cpu_baseline leg; rank 0 only)
# --------------------------------------------------------------------------

def cpu_context(A, x, info, create_s):
    """SURVEY §8(d) D5 items 2 and 3, context beside the oracle baseline:
    an OpenMP fp64 CSR SpMV on every core of the process (whole matrix, best
    of 3; not the oracle), and the oracle's single-threaded tiler on a
    bounded row slice next to the GPU tiler (create) per million nonzeros
    (the Fig. 11 analogue)."""
    from oracle import oracle as O
    out = {}
    try:
        model = next((l.split(":", 1)[1].strip() for l in open("/proc/cpuinfo") if l.startswith("model name")), "")
    except OSError:
        model = ""
    best = float("inf")
    threads = 0
    for _ in range(3):
        t = time.perf_counter()
        _, threads = O.cpu_csr_omp(A, x)
        best = min(best, time.perf_counter() - t)
    out["omp_csr"] = {"value": 2.0 * A.nnz / best / 1e9, "unit": UNIT, "cores": threads,
                      "affinity_cores": len(os.sched_getaffinity(0)), "cpu": model,
                      "kind": "openmp row-parallel fp64 CSR (not the oracle)",
                      "sample": "whole matrix, best of 3 passes"}
    rowlen = np.diff(A.rowptr.astype(np.int64))
    r1 = int(min(A.m, max(16, np.searchsorted(np.cumsum(rowlen), 2_000_000) // 16 * 16 + 16)))
    S = A.row_slice(0, r1)
    t = time.perf_counter()
    O.tile(S, {0: "ADPT", 1: "DEFERRED", 3: "FORCE_CSR"}.get(int(info.get("mode", 1)), "DEFERRED"))
    dt = time.perf_counter() - t
    out["tiler"] = {"oracle_s_per_Mnnz": dt / max(S.nnz, 1) * 1e6, "oracle_sample_nnz": int(S.nnz),
                    "gpu_create_s_per_Mnnz": create_s / max(A.nnz, 1) * 1e6,
                    "note": "oracle tiler: one thread, first rows of the matrix; GPU: tilespmv_create_from_csr"}
    return out


def oracle_sample(A, x, seconds: float, rng, max_rows=None):
    """Times the oracle (oracle/oracle.c, long-double Alg. 1, 1 thread) on a
    bounded sample of rows of A: contiguous blocks at random offsets, sized
    from a short probe to about `seconds` of CPU work.  Returns
    (GFLOP/s, rows, yref, absy, description)."""
    from oracle import oracle as O
    rowlen = np.diff(A.rowptr.astype(np.int64))
    probe = np.arange(min(A.m, 20000))
    t = time.perf_counter()
    O.spmv(A, x, probe)
    dt = max(time.perf_counter() - t, 1e-6)
    rate = max(rowlen[probe].sum(), 1) / dt                  # nnz / s
    want_nnz = int(rate * seconds)
    blocks, got = [], 0
    while got < want_nnz and got < A.nnz:
        r0 = int(rng.integers(0, max(1, A.m - 4096)))
        blk = np.arange(r0, min(A.m, r0 + 4096))
        blocks.append(blk)
        got += int(rowlen[blk].sum())
        if max_rows and sum(len(b) for b in blocks) >= max_rows:
            break
    rows = np.unique(np.concatenate(blocks)) if blocks else np.arange(min(A.m, 1))
    nnz = int(rowlen[rows].sum())
    # repeat the sample until about `seconds` of CPU work (at most 3x that)
    passes, t = 0, time.perf_counter()
    while True:
        yref, absy = O.spmv(A, x, rows)
        passes += 1
        dt = time.perf_counter() - t
        if dt >= seconds or dt * (passes + 1) / passes > 3 * seconds:
            break
    desc = (f"{rows.size} rows ({nnz} nnz, {100.0 * nnz / max(A.nnz, 1):.2f}% of the matrix) "
            f"in 4096-row blocks at seeded random offsets; {passes} pass(es), {dt:.2f} s")
    nnz *= passes
    return 2.0 * nnz / dt / 1e9, rows, yref, absy, desc, dt


# --------------------------------------------------------------------------
# reference arm: the oracle, as it stands, on the host cores
# --------------------------------------------------------------------------

def run_reference(args):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    from oracle import oracle as O
    from synthetic import gen
    A, m, n, _ = build_local(args.workload, 0, 1)
    x = gen.dense_x(n, 101)
    rng = np.random.default_rng(1234)
    # each step: the oracle over a bounded sample, sized so that warmup+steps
    # finish within ~2 minutes
    budget = 120.0 / max(1, args.steps + args.warmup)
    rowlen = np.diff(A.rowptr.astype(np.int64))
    probe = np.arange(min(A.m, 20000))
    t = time.perf_counter()
    O.spmv(A, x, probe)
    rate = max(rowlen[probe].sum(), 1) / max(time.perf_counter() - t, 1e-6)
    k = max(1, int(rate * min(budget, 2.0)))
    r0 = int(rng.integers(0, max(1, A.m - 1)))
    rows = []
    acc = 0
    r = r0
    while acc < k and len(rows) < A.m:
        rows.append(r)
        acc += rowlen[r]
        r = (r + 1) % A.m
    rows = np.array(sorted(rows))
    nnz = int(rowlen[rows].sum())
    for _ in range(args.warmup):
        O.spmv(A, x, rows)
    t = time.perf_counter()
    for _ in range(args.steps):
        O.spmv(A, x, rows)
    dt = (time.perf_counter() - t) / args.steps
    val = 2.0 * nnz / dt / 1e9
    sample = f"{rows.size} contiguous rows ({nnz} nnz) per step of {args.workload}"
    out = {"metric": METRIC, "value": val, "unit": UNIT, "n_gpus": args.gpus, "steps": args.steps,
           "warmup": args.warmup, "ms_per_step": dt * 1e3, "higher_is_better": True,
           "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
           "impl": "reference",
           "config": {"workload": args.workload, "desc": WORKLOAD_DESC.get(args.workload, ""),
                      "mode": args.mode},
           "cpu_baseline": {"value": val, "unit": UNIT, "cores": 1, "kind": "oracle",
                            "sample": sample},
           "e2e": {"value": val, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(out), flush=True)
    return 0


# --------------------------------------------------------------------------
# our arm
# --------------------------------------------------------------------------

def measure_workload(workload, mode, steps, warmup, dev, rank, P, group, cpu_seconds,
                     want_cpu, want_e2e, e2e_steps, use_graph=True):
    import torch
    from paper_conf_ipps_niuldj0t21_b200 import TiledMatrix
    from synthetic import gen

    t0 = time.perf_counter()
    assert P == 1, "measure_workload is the N = 1 path"
    A, m, n, bounds = build_local(workload, rank, P)
    log(f"[rank {rank}] {workload}: local {A.m}x{A.n} nnz {A.nnz} generated in "
        f"{time.perf_counter() - t0:.1f}s")
    x_h = gen.dense_x(n, 101)
    stream = torch.cuda.current_stream(dev)
    rp = torch.from_numpy(A.rowptr).to(dev)
    ci = torch.from_numpy(A.colidx).to(dev)
    va = torch.from_numpy(A.val).to(dev)
    torch.cuda.synchronize(dev)
    t = time.perf_counter()
    M0 = TiledMatrix.from_csr(rp, ci, va, A.m, A.n, mode=mode)
    create_s = time.perf_counter() - t
    info = M0.info()
    L2 = torch.cuda.get_device_properties(dev).L2_cache_size
    reps = max(1, -(-4 * L2 // max(info["alg_bytes"], 1)))
    mats = [M0] + [TiledMatrix.from_csr(rp, ci, va, A.m, A.n, mode=mode) for _ in range(reps - 1)]
    del rp, ci, va
    xs = [torch.from_numpy(x_h).to(dev) for _ in range(reps)]
    ys = [torch.empty(A.m, dtype=torch.float64, device=dev) for _ in range(reps)]
    def step(i):
        j = i % reps
        mats[j].run(xs[j], ys[j])

    # a step is exactly one kernel launch; the K launches go back to back
    # (programmatic dependent launch overlaps one kernel's prologue with the
    # previous one's tail) between two events, so the kernel's average launch
    # duration is the timed region / K.
    start, end = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    # N = 1: the K timed launches are captured once into a CUDA graph and
    # replayed, so the host's per-launch cost (Python + ctypes, ~8-11 us) cannot
    # starve a kernel that runs for a few microseconds.  Each graph node is one
    # launch of the SpMV kernel through tilespmv_run (PDL edges kept).
    graph, launch_mode = None, "eager"
    if use_graph:
        for i in range(warmup):
            step(i)
        torch.cuda.synchronize(dev)
        try:
            graph = torch.cuda.CUDAGraph()
            with torch.cuda.graph(graph):
                for i in range(steps):
                    mats[i % reps].run(xs[i % reps], ys[i % reps])
            graph.replay()  # upload + one untimed pass
            torch.cuda.synchronize(dev)
            launch_mode = "cuda_graph"
        except Exception as e:  # pragma: no cover
            log("graph capture failed, timing eager launches:", e)
            graph = None
    sampler = ClockSampler(dev.index if dev.index is not None else 0)
    with sampler:
        for i in range(warmup):
            step(i)
        torch.cuda.synchronize(dev)
        h0 = time.perf_counter()
        start.record(stream)
        for i in range(steps if graph is None else 0):
            step(i)
        if graph is not None:
            graph.replay()
        end.record(stream)
        h1 = time.perf_counter()
        torch.cuda.synchronize(dev)
        sampler.window(h0, time.perf_counter())
    host_launch_us = (h1 - h0) / steps * 1e6  # host time to enqueue one step
    torch.cuda.synchronize(dev)
    total_ms = start.elapsed_time(end)
    kern_ms = np.array([total_ms / steps])
    kern_max = float(np.mean(kern_ms))
    nnz_total = A.nnz
    ms_per_step = total_ms / steps
    value = 2.0 * nnz_total / (ms_per_step * 1e-3) / 1e9
    peak, peak_src = hbm_peak()
    achieved = info["alg_bytes"] / (float(np.mean(kern_ms)) * 1e-3) / 1e9
    grid, block, smem = M0.launch_shape()
    res = {"value": value, "ms_per_step": ms_per_step, "info": info, "reps": reps,
           "launch": {"grid": grid, "block": block, "smem_bytes": smem},
           "kernel_ms_mean": float(np.mean(kern_ms)), "kernel_ms_median": float(np.median(kern_ms)),
           "kernel_ms_max_over_ranks": kern_max, "create_s": create_s,
           "clocks": sampler.summary(), "nnz": nnz_total, "m": m, "n": n,
           "host_enqueue_us_per_step": host_launch_us, "launch_mode": launch_mode,
           "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                        "frac": achieved / peak, "traffic": profile_traffic(workload, mode),
                        "peak_source": peak_src,
                        "alg_bytes_per_launch": info["alg_bytes"],
                        "kernel": M0.kernel_name()}}
    # ---- correctness on the oracle's sample + CPU baseline (rank 0, N = 1)
    if want_cpu and rank == 0:
        rng = np.random.default_rng(4321)
        val, rows, yref, absy, desc, dt = oracle_sample(A, x_h, cpu_seconds, rng)
        y = ys[0].cpu().numpy()
        err = np.abs(y[rows] - yref)
        ok = bool(np.all(err <= 1e-12 * absy + 1e-300))
        res["cpu_baseline"] = {"value": val, "unit": UNIT, "cores": 1, "kind": "oracle",
                               "sample": desc}
        res["parity"] = {"rows_checked": int(rows.size), "ok": ok,
                         "max_err_over_absy": float(np.max(err / (absy + 1e-300))) if rows.size else 0.0,
                         "tolerance": "1e-12*sum|a_ij x_j| + 1e-300"}
        res["cpu_context"] = cpu_context(A, x_h, info, create_s)
    # ---- end to end through the host-buffer C-ABI call
    if want_e2e:
        hx = torch.from_numpy(x_h).pin_memory()
        hy = torch.empty(A.m, dtype=torch.float64).pin_memory()
        for _ in range(2):
            M0.run_host(hx, hy)
        torch.cuda.synchronize(dev)
        t = time.perf_counter()
        for _ in range(e2e_steps):
            M0.run_host(hx, hy)
        e2e_s = (time.perf_counter() - t) / e2e_steps
        res["e2e"] = {"value": 2.0 * nnz_total / e2e_s / 1e9, "unit": UNIT,
                      "h2d_bytes_per_step": 8 * n, "d2h_bytes_per_step": 8 * A.m,
                      "ms_per_step": e2e_s * 1e3, "steps": e2e_steps,
                      "call": "tilespmv_run_host (pinned host x -> H2D -> kernel -> D2H y -> sync)"}
    for M in mats:
        M.close()
    return res


def measure_sharded(workload, mode, steps, warmup, dev, rank, P, group, exchange, e2e_steps):
    """N > 1: tile-row shards (x replicated at start), one step = the rank's
    SpMV plus the exchange that makes x_{k+1} available where it is needed:
      halo      -- neighbour-only NCCL send/recv of the x rows each peer's
                   columns touch, overlapped with the interior SpMV; the
                   boundary SpMVs run after it lands;
      allgather -- the SpMV of all local rows, then an NCCL all-gather of y
                   (SURVEY 8(e)).
    x stays fixed across steps (the exchanged rows equal what is there), so
    the timed work is exactly one iteration's and values stay finite.  Times
    are device events on the compute stream, max over ranks."""
    import torch
    import torch.distributed as dist
    from paper_conf_ipps_niuldj0t21_b200 import TiledMatrix
    from paper_conf_ipps_niuldj0t21_b200.sharded import HaloSpMV, plan_halo
    from synthetic import gen

    t0 = time.perf_counter()
    A, m, n, bounds = build_local(workload, rank, P)
    a, b = bounds[rank], bounds[rank + 1]
    log(f"[rank {rank}] {workload}: rows [{a},{b}) nnz {A.nnz} generated in {time.perf_counter() - t0:.1f}s")
    x_h = gen.dense_x(n, 101)
    stream = torch.cuda.current_stream(dev)
    x = torch.from_numpy(x_h).to(dev)
    torch.cuda.synchronize(dev)
    t = time.perf_counter()
    if exchange == "halo":
        plan = plan_halo(A.rowptr, A.colidx, bounds, rank, P, group)
        parts = plan.parts
    else:
        plan, parts = None, [(a, b, True)]
    mats = []
    for r0, r1, _ in parts:
        S = A.row_slice(r0 - a, r1 - a)
        mats.append(TiledMatrix.from_csr(torch.from_numpy(S.rowptr).to(dev), torch.from_numpy(S.colidx).to(dev),
                                         torch.from_numpy(S.val).to(dev), S.m, S.n, mode=mode))
    torch.cuda.synchronize(dev)
    create_s = time.perf_counter() - t
    infos = [M.info() for M in mats]
    dom = max(range(len(mats)), key=lambda i: infos[i]["alg_bytes"])  # dominant kernel
    maxrows = max(bounds[i + 1] - bounds[i] for i in range(P))
    y = torch.empty(n if exchange == "halo" else P * maxrows, dtype=torch.float64, device=dev)
    kev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(steps)]

    if exchange == "halo":
        def mk(M):
            return lambda xf, yo: M.run(xf, yo)
        H = HaloSpMV(plan, [mk(M) for M in mats], group=group,
                     host_staging=os.environ.get("TILESPMV_BENCH_ONE_GPU") == "1")
        ev_slot = [None]

        def timed(xf, yo, M=mats[dom]):
            e = ev_slot[0]
            if e is not None:
                e[0].record(stream)
            M.run(xf, yo)
            if e is not None:
                e[1].record(stream)
        H.spmvs[dom] = timed

        def step(i, ev=None):
            ev_slot[0] = ev
            H.step(x, y)
    else:
        def step(i, ev=None):
            yl = y[rank * maxrows: rank * maxrows + (b - a)]
            if ev is not None:
                ev[0].record(stream)
            mats[0].run(x, yl)
            if ev is not None:
                ev[1].record(stream)
            dist.all_gather_into_tensor(y, y[rank * maxrows:(rank + 1) * maxrows], group=group)

    start, end = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    sampler = ClockSampler(dev.index if dev.index is not None else 0)
    with sampler:
        for i in range(warmup):
            step(i)
        torch.cuda.synchronize(dev)
        dist.barrier(group=group)
        torch.cuda.synchronize(dev)
        h0 = time.perf_counter()
        start.record(stream)
        for i in range(steps):
            step(i, kev[i])
        end.record(stream)
        torch.cuda.synchronize(dev)
        sampler.window(h0, time.perf_counter())
    dist.barrier(group=group)
    total_ms = start.elapsed_time(end)
    kern_ms = np.array([e0.elapsed_time(e1) for e0, e1 in kev])
    t_ = torch.tensor([total_ms, float(np.mean(kern_ms))], dtype=torch.float64, device=dev)
    dist.all_reduce(t_, op=dist.ReduceOp.MAX, group=group)
    total_ms, kern_max = float(t_[0]), float(t_[1])
    t_ = torch.tensor([A.nnz], dtype=torch.int64, device=dev)
    dist.all_reduce(t_, group=group)
    nnz_total = int(t_[0])
    ms_per_step = total_ms / steps
    peak, peak_src = hbm_peak()
    achieved = infos[dom]["alg_bytes"] / (float(np.mean(kern_ms)) * 1e-3) / 1e9
    grid, block, smem = mats[dom].launch_shape()
    res = {"value": 2.0 * nnz_total / (ms_per_step * 1e-3) / 1e9, "ms_per_step": ms_per_step,
           "info": infos[dom], "reps": 1, "nnz": nnz_total, "m": m, "n": n, "create_s": create_s,
           "launch": {"grid": grid, "block": block, "smem_bytes": smem},
           "kernel_ms_mean": float(np.mean(kern_ms)), "kernel_ms_median": float(np.median(kern_ms)),
           "kernel_ms_max_over_ranks": kern_max, "clocks": sampler.summary(),
           "host_enqueue_us_per_step": None, "launch_mode": "eager",
           "launches_per_step": len(mats),
           "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                        "frac": achieved / peak, "traffic": None, "peak_source": peak_src,
                        "alg_bytes_per_launch": infos[dom]["alg_bytes"],
                        "kernel": mats[dom].kernel_name() + (" (interior part)" if exchange == "halo" else "")}}
    if exchange == "halo":
        res["exchange"] = {"kind": "halo (NCCL send/recv, overlapped with the interior SpMV)",
                           "recv_bytes_rank0": 8 * plan.recv_elems, "send_bytes_rank0": 8 * plan.send_elems,
                           "parts_rank0": [[r0, r1, bool(it)] for r0, r1, it in parts]}
    else:
        res["exchange"] = {"kind": "NCCL all-gather of y", "bytes_per_rank": 8 * P * maxrows}
    # ---- end to end: per step every rank copies its own x rows in (pinned
    # host -> device), runs the step, and reads its own y rows back
    if e2e_steps > 0:
        hx = torch.from_numpy(x_h[a:b].copy()).pin_memory()
        hy = torch.empty(b - a, dtype=torch.float64).pin_memory()

        def e2e_step():
            x[a:b].copy_(hx, non_blocking=True)
            step(0)
            hy.copy_(y[a:b] if exchange == "halo" else y[rank * maxrows: rank * maxrows + (b - a)],
                     non_blocking=True)
            stream.synchronize()

        for _ in range(2):
            e2e_step()
        dist.barrier(group=group)
        t = time.perf_counter()
        for _ in range(e2e_steps):
            e2e_step()
        e2e_s = torch.tensor([(time.perf_counter() - t) / e2e_steps], dtype=torch.float64, device=dev)
        dist.all_reduce(e2e_s, op=dist.ReduceOp.MAX, group=group)
        e2e_s = float(e2e_s[0])
        res["e2e"] = {"value": 2.0 * nnz_total / e2e_s / 1e9, "unit": UNIT,
                      "h2d_bytes_per_step": 8 * n, "d2h_bytes_per_step": 8 * m,
                      "ms_per_step": e2e_s * 1e3, "steps": e2e_steps,
                      "call": "per rank: H2D own x rows -> step (exchange + SpMV) -> D2H own y rows; "
                              "bytes summed over ranks, time max over ranks"}
    for M in mats:
        M.close()
    return res


def run_ours(args):
    import torch
    import torch.distributed as dist
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    P = max(world, 1)
    if P != args.gpus:
        log(f"warning: --gpus {args.gpus} but WORLD_SIZE {P}")
    group = None
    # development hook: TILESPMV_BENCH_ONE_GPU=1 runs every rank on cuda:0 over
    # gloo (exercises the N > 1 code path on a one-GPU box; not a bench number)
    one_gpu = os.environ.get("TILESPMV_BENCH_ONE_GPU") == "1"
    dev = torch.device("cuda", 0 if one_gpu else local)
    torch.cuda.set_device(dev)
    if P > 1:
        if one_gpu:
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=dev)
        group = dist.group.WORLD
    if P > 1:
        res = measure_sharded(args.workload, args.mode, args.steps, args.warmup, dev, rank, P, group,
                              args.exchange, args.e2e_steps)
    else:
        res = measure_workload(args.workload, args.mode, args.steps, args.warmup, dev, rank, P, group,
                               args.cpu_seconds, want_cpu=not args.no_cpu_baseline,
                               want_e2e=True, e2e_steps=args.e2e_steps, use_graph=not args.no_graph)
    secondary = {}
    if P == 1 and not args.no_secondary and args.workload != "fem":
        r2 = measure_workload("fem", args.mode, max(args.steps, 200), args.warmup, dev, 0, 1, None,
                              2.0, want_cpu=False, want_e2e=False, e2e_steps=0, use_graph=not args.no_graph)
        secondary["fem"] = {"value": r2["value"], "unit": UNIT, "ms_per_step": r2["ms_per_step"],
                            "host_enqueue_us_per_step": r2["host_enqueue_us_per_step"],
                            "launch_mode": r2["launch_mode"],
                            "roofline": r2["roofline"], "replicas_rotated": r2["reps"],
                            "desc": WORKLOAD_DESC["fem"]}
    if rank == 0:
        info = res["info"]
        out = {"metric": METRIC, "value": res["value"], "unit": UNIT, "n_gpus": P,
               "steps": args.steps, "warmup": args.warmup, "ms_per_step": res["ms_per_step"],
               "higher_is_better": True, "scaling": "strong" if P > 1 else "weak",
               "vs_baseline": None, "dtype": "f64", "data": "synthetic",
               "config": {"workload": args.workload, "desc": WORKLOAD_DESC.get(args.workload, ""),
                          "mode": args.mode, "m": res["m"], "n": res["n"], "nnz": res["nnz"],
                          "parallelism": f"tile-row shards x{P}" if P > 1 else "1 GPU",
                          "l2": ("inputs larger than L2" if res["reps"] == 1 else
                                 f"rotating {res['reps']} replicas (> 4x L2)"),
                          "step": (("halo exchange overlapped with the interior SpMV + boundary SpMVs"
                                    if args.exchange == "halo" else "SpMV + NCCL all-gather of y")
                                   if P > 1 else "one SpMV launch"),
                          "launch_mode": res["launch_mode"],
                          "numtile": info["numtile"], "rem_nnz": info["rem_nnz"],
                          "kept_tiles": dict(zip(["CSR", "COO", "ELL", "HYB", "DNS", "DNSROW", "DNSCOL"],
                                                 info["kept_tiles"])),
                          "alg_bytes_per_spmv": info["alg_bytes"], "create_s": res["create_s"]},
               "roofline": res["roofline"],
               "cpu_baseline": res.get("cpu_baseline"),
               "e2e": res.get("e2e"),
               "gpu_launches": args.steps,
               "kernel_ms": {"mean": res["kernel_ms_mean"], "median": res["kernel_ms_median"],
                             "max_over_ranks": res["kernel_ms_max_over_ranks"]},
               "clocks": res["clocks"],
               "host_enqueue_us_per_step": res["host_enqueue_us_per_step"],
               "launch": res["launch"],
               "parity": res.get("parity")}
        if res.get("cpu_context"):
            out["cpu_context"] = res["cpu_context"]
        if "exchange" in res:
            out["exchange"] = res["exchange"]
            out["gpu_launches"] = args.steps * res["launches_per_step"]
        if secondary:
            out["secondary"] = secondary
        print(json.dumps(out), flush=True)
    if P > 1:
        dist.destroy_process_group()
    return 0


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=300)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--workload", default=DEFAULT_WORKLOAD)
    ap.add_argument("--mode", default="DEFERRED", choices=["ADPT", "DEFERRED", "AUTO", "FORCE_CSR"])
    ap.add_argument("--cpu-seconds", type=float, default=10.0)
    ap.add_argument("--exchange", default="halo", choices=["halo", "allgather"],
                    help="N>1: neighbour-only x exchange (default) or all-gather of y")
    ap.add_argument("--e2e-steps", type=int, default=20)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-secondary", action="store_true")
    ap.add_argument("--no-graph", action="store_true",
                    help="N=1: time K eager launches instead of one CUDA-graph replay of them")
    args = ap.parse_args()
    assert args.warmup >= 3, "the contract requires >= 3 warm-up steps"
    if args.impl == "reference":
        return run_reference(args)
    return run_ours(args)


if __name__ == "__main__":
    sys.exit(main())
