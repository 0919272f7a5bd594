#!/usr/bin/env python
"""Benchmark of the B200 tiled fp64 SpMV hot path (TileSpMV, IPDPS'21).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]
                    [--workload stencil27_200|fem|rmat20|mixed|lap2d_64] [--mode DEFERRED]

One "step" is one pass of the whole hot path over one batch of synthetic input:
the single-kernel tiled SpMV y = A x (N = 1), or, tile-row sharded over N
GPUs, each rank's SpMV of its tile rows followed by the NCCL all-gather of y
(N > 1, the north star's exchange; the halo exchange of SURVEY §8(f) f1 is
timed beside it).  The matrix is built once (GPU tiler, not timed).  Inputs
are resident in HBM when the timed region starts; working sets smaller than
4x L2 rotate over independent replicas so every step streams from HBM.

Prints ONE JSON line on rank 0 (the driver contract): metric/value/unit,
roofline of the SpMV kernel against MEASURED_PEAKS.json, the CPU oracle
baseline, an end-to-end number through the host-buffer C-ABI call, clocks,
and (N = 1) every other BASELINE config as a `secondary` entry, each with its
pipelined and single-launch timing.
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
# N = 1: the other BASELINE configs, each its own line in `secondary`
SECONDARY = [("fem", "DEFERRED"), ("rmat20", "DEFERRED"), ("mixed", "ADPT"), ("mixed", "DEFERRED"),
             ("lap2d_64", "DEFERRED"),
             # the optional byte-cost selection mode (not the paper's rule)
             ("fem", "BYTES")]
SINGLE_LAUNCHES = 60  # single-launch timing: median of this many isolated launches
CHUNKS = 4            # N > 1, --exchange chunked: chunks per rank


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


def run_config(args, m, n, nnz, P):
    """The `config` object of the JSON line: the same keys and values in both
    arms (ours and --impl reference), so the driver can match them."""
    return {"workload": args.workload, "desc": WORKLOAD_DESC.get(args.workload, ""), "mode": args.mode,
            "m": int(m), "n": int(n), "nnz": int(nnz),
            "parallelism": f"tile-row shards x{P}" if P > 1 else "1 GPU",
            "l2": "inputs larger than L2 or rotated over replicas > 4x L2 (GPU arm)"}


# --------------------------------------------------------------------------
# CPU legs (rank 0 only): the oracle baseline and context
# --------------------------------------------------------------------------

def oracle_f64_baseline(A, x, passes: int = 5):
    """cpu_baseline: the plain fp64 row loop of the
    oracle (oracle_spmv_f64, Alg. 1 in double, one thread) over the whole
    matrix, best of `passes`."""
    from oracle import oracle as O
    best = float("inf")
    for _ in range(passes):
        t = time.perf_counter()
        O.spmv_f64(A, x)
        best = min(best, time.perf_counter() - t)
    return {"value": 2.0 * A.nnz / best / 1e9, "unit": UNIT, "cores": 1, "kind": "oracle",
            "sample": f"whole matrix ({A.nnz} nnz), best of {passes} passes, "
                      f"oracle_spmv_f64 (Alg. 1 in fp64, one thread); {best:.3f} s per pass"}


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


def parity_rows(A, x, y, rng, nrows: int = 400_000):
    """North-star check of y on a bounded row sample (first/last rows, the
    longest rows, and 4096-row blocks at seeded offsets) against the
    extended-precision oracle."""
    from oracle import oracle as O
    rowlen = np.diff(A.rowptr.astype(np.int64))
    parts = [np.arange(min(64, A.m)), np.arange(max(0, A.m - 64), A.m), np.argsort(rowlen)[-64:]]
    got = 0
    while got < nrows and got < A.m:
        r0 = int(rng.integers(0, max(1, A.m - 4096)))
        parts.append(np.arange(r0, min(A.m, r0 + 4096)))
        got += 4096
    rows = np.unique(np.concatenate(parts))
    yref, absy = O.spmv(A, x, rows)
    err = np.abs(y[rows] - yref)
    return {"rows_checked": int(rows.size), "ok": bool(np.all(err <= 1e-12 * absy + 1e-300)),
            "max_err_over_absy": float(np.max(err / (absy + 1e-300))) if rows.size else 0.0,
            "tolerance": "1e-12*sum|a_ij x_j| + 1e-300"}


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
    # a step is one oracle_spmv_f64 pass over the whole matrix, unless the
    # whole run would exceed ~150 s: then a contiguous row block per step
    t = time.perf_counter()
    O.spmv_f64(A, x)
    one = time.perf_counter() - t
    S, sample = A, f"whole matrix ({A.nnz} nnz) per step"
    if one * (args.steps + args.warmup) > 150.0:
        frac = 150.0 / (one * (args.steps + args.warmup))
        r1 = max(16, int(A.m * frac) // 16 * 16)
        S = A.row_slice(0, r1)
        sample = f"rows [0, {r1}) ({S.nnz} nnz, {100.0 * S.nnz / A.nnz:.1f}% of the matrix) per step"
    for _ in range(args.warmup):
        O.spmv_f64(S, x)
    t = time.perf_counter()
    for _ in range(args.steps):
        O.spmv_f64(S, x)
    dt = (time.perf_counter() - t) / args.steps
    val = 2.0 * S.nnz / dt / 1e9
    sample += "; oracle_spmv_f64 (Alg. 1 in fp64, one thread)"
    out = {"metric": METRIC, "value": val, "unit": UNIT, "n_gpus": args.gpus, "steps": args.steps,
           "warmup": args.warmup, "ms_per_step": dt * 1e3, "higher_is_better": True,
           "scaling": "strong" if args.gpus > 1 else "weak", "vs_baseline": None, "dtype": "f64",
           "data": "synthetic", "impl": "reference",
           "config": run_config(args, m, n, A.nnz, args.gpus),
           "cpu_baseline": {"value": val, "unit": UNIT, "cores": 1, "kind": "oracle", "sample": sample},
           "e2e": {"value": val, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(out), flush=True)
    return 0


# --------------------------------------------------------------------------
# our arm
# --------------------------------------------------------------------------

def time_pipelined(launch, steps, warmup, dev, use_graph=True, sample_clocks=True):
    """K launches back to back (launch(i) enqueues step i), captured once in a
    CUDA graph and replayed (the host's per-launch cost, ~8-11 us of Python +
    ctypes, cannot starve a kernel of a few microseconds), timed with CUDA
    events on the launching stream.  Programmatic dependent launch overlaps
    each kernel's prologue with the previous one's tail.  Returns
    (ms per step, launch mode, host enqueue us per step, clocks)."""
    import torch
    stream = torch.cuda.current_stream(dev)
    graph, mode = None, "eager"
    if use_graph:
        for i in range(warmup):
            launch(i)
        torch.cuda.synchronize(dev)
        try:
            graph = torch.cuda.CUDAGraph()
            with torch.cuda.graph(graph):
                for i in range(steps):
                    launch(i)
            graph.replay()  # upload + one untimed pass
            torch.cuda.synchronize(dev)
            mode = "cuda_graph"
        except Exception as e:  # pragma: no cover
            log("graph capture failed, timing eager launches:", e)
            graph = None
    start, end = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    sampler = ClockSampler(dev.index if dev.index is not None else 0) if sample_clocks else None
    if sampler:
        sampler.__enter__()
    try:
        for i in range(warmup):
            launch(i)
        torch.cuda.synchronize(dev)
        h0 = time.perf_counter()
        start.record(stream)
        if graph is not None:
            graph.replay()
        else:
            for i in range(steps):
                launch(i)
        end.record(stream)
        h1 = time.perf_counter()
        torch.cuda.synchronize(dev)
        if sampler:
            sampler.window(h0, time.perf_counter())
    finally:
        if sampler:
            sampler.__exit__()
    return start.elapsed_time(end) / steps, mode, (h1 - h0) / steps * 1e6, sampler.summary() if sampler else None


def time_single(launch, dev, reps, n=SINGLE_LAUNCHES):
    """Isolated launches: an event pair around ONE launch with no kernel of
    ours before it (no PDL overlap with a predecessor), replicas rotated.
    The stream is held by a ~0.2 ms spin kernel while the event, the launch
    and the second event are enqueued, so the pair times the device, not the
    host's Python enqueue.  Two ways to launch: `eager` (tilespmv_run, a
    cudaLaunchKernelEx from the host) and `graph` (the same call captured as
    a one-node CUDA graph per replica, replayed).  Returns median / p10 /
    p90 ms of each.  The same pair around a 1-element torch kernel gives the floor of this
    measurement (`launch_floor_ms`: launch latency and event overhead with no
    work)."""
    import torch
    stream = torch.cuda.current_stream(dev)
    tiny = torch.zeros(1, device=dev)
    graphs = []
    for j in range(reps):
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g):
            launch(j)
        graphs.append(g)
    tg = torch.cuda.CUDAGraph()
    with torch.cuda.graph(tg):
        tiny.add_(1.0)
    torch.cuda.synchronize(dev)
    out = {}
    for kind in ("eager", "graph"):
        ts, fs = [], []
        for i in range(n + 3):
            for what, acc in (("spmv", ts), ("tiny", fs)):
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                torch.cuda.synchronize(dev)
                torch.cuda._sleep(400_000)
                e0.record(stream)
                if what == "tiny":
                    tg.replay() if kind == "graph" else tiny.add_(1.0)
                elif kind == "graph":
                    graphs[i % reps].replay()
                else:
                    launch(i)
                e1.record(stream)
                torch.cuda.synchronize(dev)
                if i >= 3:
                    acc.append(e0.elapsed_time(e1))
        t = np.array(ts)
        out[kind] = {"median_ms": float(np.median(t)), "p10_ms": float(np.percentile(t, 10)),
                     "p90_ms": float(np.percentile(t, 90)), "launches": n,
                     "launch_floor_ms": float(np.median(fs))}
    return out


def measure_workload(A, x_h, mode, steps, warmup, dev, use_graph=True, single=True, e2e_steps=0,
                     check=True, sample_clocks=True):
    """One N = 1 workload: pipelined per-launch time (the step), single-launch
    time, roofline, parity on sampled rows, optional e2e through the host
    C-ABI call."""
    import torch
    from paper_conf_ipps_niuldj0t21_b200 import TiledMatrix
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

    def launch(i):
        j = i % reps
        mats[j].run(xs[j], ys[j])

    ms, lmode, enq_us, clocks = time_pipelined(launch, steps, warmup, dev, use_graph, sample_clocks)
    peak, peak_src = hbm_peak()
    achieved = info["alg_bytes"] / (ms * 1e-3) / 1e9
    res = {"value": 2.0 * A.nnz / (ms * 1e-3) / 1e9, "ms_per_step": ms, "info": info, "reps": reps,
           "launch_mode": lmode, "host_enqueue_us_per_step": enq_us, "clocks": clocks, "create_s": create_s,
           "launch": dict(zip(("grid", "block", "smem_bytes"), M0.launch_shape())),
           "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                        "frac": achieved / peak, "traffic": profile_traffic(A.name, mode),
                        "peak_source": peak_src, "alg_bytes_per_launch": info["alg_bytes"],
                        "kernel": M0.kernel_name(),
                        "timing": f"pipelined: {steps} back-to-back launches (PDL) / {steps}"}}
    if single:
        s = time_single(launch, dev, reps)
        for v in s.values():
            v["achieved_gbs"] = info["alg_bytes"] / (v["median_ms"] * 1e-3) / 1e9
            v["frac"] = v["achieved_gbs"] / peak
            v["gflops"] = 2.0 * A.nnz / (v["median_ms"] * 1e-3) / 1e9
        s["note"] = ("one launch between events, no kernel of ours before it: includes the front-end launch "
                     "latency and the cold prologue that PDL hides in back-to-back runs; launch_floor_ms is the "
                     "same measurement of a 1-element torch kernel")
        res["single_launch"] = s
    if check:
        torch.cuda.synchronize(dev)
        res["parity"] = parity_rows(A, x_h, ys[0].cpu().numpy(), np.random.default_rng(4321))
    if e2e_steps > 0:
        hx = torch.from_numpy(x_h).pin_memory()
        hy = torch.empty(A.m, dtype=torch.float64).pin_memory()
        for _ in range(2):
            M0.run_host(hx, hy)
        torch.cuda.synchronize(dev)
        t = time.perf_counter()
        for _ in range(e2e_steps):
            M0.run_host(hx, hy)
        e2e_s = (time.perf_counter() - t) / e2e_steps
        res["e2e"] = {"value": 2.0 * A.nnz / e2e_s / 1e9, "unit": UNIT,
                      "h2d_bytes_per_step": 8 * A.n, "d2h_bytes_per_step": 8 * A.m,
                      "ms_per_step": e2e_s * 1e3, "steps": e2e_steps,
                      "call": "tilespmv_run_host (pinned host x -> H2D -> kernel -> D2H y -> sync)",
                      "note": f"serial PCIe round trip: the {8 * (A.n + A.m) / 1e6:.0f} MB of x and y copies "
                              f"dominate; the kernel is {ms:.3f} ms of it"}
    for M in mats:
        M.close()
    return res


def secondary_entry(r, workload, mode):
    out = {"workload": workload, "mode": mode, "desc": WORKLOAD_DESC.get(workload, ""),
           "value": r["value"], "unit": UNIT, "ms_per_step": r["ms_per_step"],
           "launch_mode": r["launch_mode"], "host_enqueue_us_per_step": r["host_enqueue_us_per_step"],
           "roofline": r["roofline"], "replicas_rotated": r["reps"], "clocks": r["clocks"],
           "nnz": r["info"]["nnz"], "rem_nnz": r["info"]["rem_nnz"], "numtile": r["info"]["numtile"],
           "kernel": r["roofline"]["kernel"]}
    for k in ("single_launch", "parity"):
        if k in r:
            out[k] = r[k]
    return out


def measure_sharded(workload, mode, steps, warmup, dev, rank, P, group, exchange, e2e_steps, one_gpu):
    """N > 1: tile-row shards (x replicated at start), one step = the rank's
    SpMV plus the exchange that makes x_{k+1} available where it is needed:
      allgather -- the SpMV of all local rows, then an NCCL all-gather of y
                   (the north star's exchange);
      halo      -- neighbour-only NCCL send/recv of the x rows each peer's
                   columns touch, overlapped with the interior SpMV; the
                   boundary SpMVs run after it lands;
      chunked   -- the all-gather in CHUNKS pieces, each rank's chunk i sent
                   to every peer (NCCL send/recv) while chunk i + 1 computes
                   (SURVEY 8(e), B200-native improvement 1);
      fused     -- no collective: the SpMV kernel stores its y rows into every
                   rank's x_{k+1} through CUDA IPC / NVLink mappings
                   (tilespmv_run_scatter), one barrier per step (SURVEY 8(e),
                   B200-native improvement 2).
    x stays fixed across steps (the exchanged rows equal what is there), so
    the timed work is exactly one iteration's and values stay finite.  Times
    are device events on the compute stream, max over ranks: the step, the
    SpMV kernels alone, and the rest (the exchange, exposed part)."""
    import torch
    import torch.distributed as dist
    from paper_conf_ipps_niuldj0t21_b200 import TiledMatrix
    from paper_conf_ipps_niuldj0t21_b200.sharded import (ChunkedAllGatherSpMV, FusedScatterSpMV, HaloSpMV,
                                                         ShardedSpMV, build_shard_handles, chunk_bounds, plan_halo)
    from synthetic import gen

    t0 = time.perf_counter()
    A, m, n, bounds = build_local(workload, rank, P)
    a, b = bounds[rank], bounds[rank + 1]
    log(f"[rank {rank}] {workload}: rows [{a},{b}) nnz {A.nnz} generated in {time.perf_counter() - t0:.1f}s")
    x_h = gen.dense_x(n, 101)
    stream = torch.cuda.current_stream(dev)
    x = torch.from_numpy(x_h).to(dev)
    torch.cuda.synchronize(dev)

    def create(sl, md, kn):
        S = A.row_slice(sl[0] - a, sl[1] - a)
        return TiledMatrix.from_csr(torch.from_numpy(S.rowptr).to(dev), torch.from_numpy(S.colidx).to(dev),
                                    torch.from_numpy(S.val).to(dev), S.m, S.n, mode=md, kernel=kn)

    t = time.perf_counter()
    if exchange == "halo":
        plan = plan_halo(A.rowptr, A.colidx, bounds, rank, P, group)
        parts = plan.parts
    elif exchange == "chunked":
        cb = chunk_bounds(bounds, CHUNKS)[rank]
        plan, parts = None, [(cb[i], cb[i + 1], True) for i in range(CHUNKS)]
    else:
        plan, parts = None, [(a, b, True)]
    mats, _, _ = build_shard_handles(create, [(r0, r1) for r0, r1, _ in parts], A.nnz, mode=mode,
                                     group=group, device=dev if not one_gpu else None)
    torch.cuda.synchronize(dev)
    create_s = time.perf_counter() - t
    infos = [M.info() for M in mats]
    dom = max(range(len(mats)), key=lambda i: infos[i]["alg_bytes"])  # dominant kernel
    # per step: [step start, spmv start/end per part..., step end]
    nev = 2 + 2 * len(mats)
    evs = [[torch.cuda.Event(enable_timing=True) for _ in range(nev)] for _ in range(steps)]
    cur = [None]

    def timed_run(i, M):
        def f(xf, yo):
            e = cur[0]
            if e is not None:
                e[1 + 2 * i].record(stream)
            M.run(xf, yo)
            if e is not None:
                e[2 + 2 * i].record(stream)
        return f

    if exchange == "fused":
        F = FusedScatterSpMV(mats[0], bounds, rank, P, x, group=group)
        Mf = mats[0]

        def step(ev=None):
            cur[0] = ev
            if ev is not None:
                ev[0].record(stream)
                ev[1].record(stream)
            # x stays fixed: every step reads buffer 0 and scatters into buffer 1
            Mf.run_scatter(F.bufs[0].tensor, F.bufs[1].tensor[a:b], F.peers[1])
            if ev is not None:
                ev[2].record(stream)
            F._barrier()
            if ev is not None:
                ev[-1].record(stream)
        y = F.bufs[1].tensor
    elif exchange in ("halo", "chunked"):
        y = torch.empty(n, dtype=torch.float64, device=dev)
        if exchange == "halo":
            H = HaloSpMV(plan, [timed_run(i, M) for i, M in enumerate(mats)], group=group, host_staging=one_gpu)
        else:
            H = ChunkedAllGatherSpMV([timed_run(i, M) for i, M in enumerate(mats)], bounds, rank, P, group=group,
                                     host_staging=one_gpu)

        def step(ev=None):
            cur[0] = ev
            if ev is not None:
                ev[0].record(stream)
            H.step(x, y)
            if ev is not None:
                ev[-1].record(stream)
    else:
        sh = ShardedSpMV(timed_run(0, mats[0]), bounds, rank, P, group=group, device=dev, host_staging=one_gpu)

        def step(ev=None):
            cur[0] = ev
            if ev is not None:
                ev[0].record(stream)
            sh.spmv(x, sh.local_out())
            sh.exchange()
            if ev is not None:
                ev[-1].record(stream)

    start, end = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    sampler = ClockSampler(dev.index if dev.index is not None else 0)
    with sampler:
        for _ in range(warmup):
            step()
        torch.cuda.synchronize(dev)
        dist.barrier(group=group)
        torch.cuda.synchronize(dev)
        h0 = time.perf_counter()
        start.record(stream)
        for i in range(steps):
            step(evs[i])
        end.record(stream)
        torch.cuda.synchronize(dev)
        sampler.window(h0, time.perf_counter())
    dist.barrier(group=group)
    total_ms = start.elapsed_time(end)
    spmv_ms = np.array([sum(e[1 + 2 * i].elapsed_time(e[2 + 2 * i]) for i in range(len(mats))) for e in evs])
    step_ms = np.array([e[0].elapsed_time(e[-1]) for e in evs])
    dom_ms = np.array([e[1 + 2 * dom].elapsed_time(e[2 + 2 * dom]) for e in evs])
    red_dev = dev if not one_gpu else torch.device("cpu")
    t_ = torch.tensor([total_ms, float(np.mean(spmv_ms)), float(np.mean(step_ms - spmv_ms)),
                       float(np.mean(dom_ms))], dtype=torch.float64, device=red_dev)
    dist.all_reduce(t_, op=dist.ReduceOp.MAX, group=group)
    total_ms, spmv_max, exch_max, dom_max = (float(v) for v in t_.cpu())
    t_ = torch.tensor([A.nnz], dtype=torch.int64, device=red_dev)
    dist.all_reduce(t_, group=group)
    nnz_total = int(t_[0])
    ms_per_step = total_ms / steps
    peak, peak_src = hbm_peak()
    achieved = infos[dom]["alg_bytes"] / (float(np.mean(dom_ms)) * 1e-3) / 1e9
    res = {"value": 2.0 * nnz_total / (ms_per_step * 1e-3) / 1e9, "ms_per_step": ms_per_step,
           "info": infos[dom], "reps": 1, "nnz": nnz_total, "m": m, "n": n, "create_s": create_s,
           "launch": dict(zip(("grid", "block", "smem_bytes"), mats[dom].launch_shape())),
           "clocks": sampler.summary(), "launch_mode": "eager", "launches_per_step": len(mats),
           "breakdown_ms_max_over_ranks": {"step": ms_per_step, "spmv_kernels": spmv_max,
                                           "exchange_exposed": exch_max, "dominant_kernel": dom_max},
           "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                        "frac": achieved / peak, "traffic": None, "peak_source": peak_src,
                        "alg_bytes_per_launch": infos[dom]["alg_bytes"],
                        "kernel": mats[dom].kernel_name() + (" (interior part)" if exchange == "halo" else "")}}
    if exchange == "fused":
        res["exchange"] = {"kind": "fused scatter epilogue (y rows stored into every rank's x_{k+1} over CUDA IPC / "
                                   "NVLink; one barrier per step, no collective)",
                           "bytes_per_rank": 8 * (b - a) * (P - 1)}
    elif exchange == "chunked":
        res["exchange"] = {"kind": f"all-gather in {CHUNKS} chunks (NCCL send/recv of chunk i while chunk i+1 "
                                   "computes)", "bytes_per_rank": 8 * (n - (b - a))}
    elif exchange == "halo":
        res["exchange"] = {"kind": "halo (NCCL send/recv, overlapped with the interior SpMV)",
                           "recv_bytes_rank": 8 * plan.recv_elems, "send_bytes_rank": 8 * plan.send_elems,
                           "parts_rank": [[r0, r1, bool(it)] for r0, r1, it in parts]}
    else:
        res["exchange"] = {"kind": "NCCL all-gather of y", "bytes_per_rank": 8 * P * sh.maxrows}
    # ---- end to end: per step every rank copies its own x rows in (pinned
    # host -> device), runs the step, and reads its own y rows back
    if e2e_steps > 0:
        hx = torch.from_numpy(x_h[a:b].copy()).pin_memory()
        hy = torch.empty(b - a, dtype=torch.float64).pin_memory()

        def e2e_step():
            x[a:b].copy_(hx, non_blocking=True)
            step()
            hy.copy_(y[a:b] if exchange in ("halo", "chunked", "fused") else sh.local_out(), non_blocking=True)
            stream.synchronize()

        for _ in range(2):
            e2e_step()
        dist.barrier(group=group)
        t = time.perf_counter()
        for _ in range(e2e_steps):
            e2e_step()
        e2e_s = torch.tensor([(time.perf_counter() - t) / e2e_steps], dtype=torch.float64, device=red_dev)
        dist.all_reduce(e2e_s, op=dist.ReduceOp.MAX, group=group)
        e2e_s = float(e2e_s[0])
        res["e2e"] = {"value": 2.0 * nnz_total / e2e_s / 1e9, "unit": UNIT,
                      "h2d_bytes_per_step": 8 * n, "d2h_bytes_per_step": 8 * m,
                      "ms_per_step": e2e_s * 1e3, "steps": e2e_steps,
                      "call": "per rank: H2D own x rows -> step (exchange + SpMV) -> D2H own y rows; "
                              "bytes summed over ranks, time max over ranks"}
    if exchange == "fused":
        F.close()
    for M in mats:
        M.close()
    return res


def run_ours(args):
    import torch
    import torch.distributed as dist
    from synthetic import gen
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
    secondary = {}
    if P > 1:
        res = measure_sharded(args.workload, args.mode, args.steps, args.warmup, dev, rank, P, group,
                              args.exchange, args.e2e_steps, one_gpu)
        if not args.no_secondary:  # the other exchange, same shards
            others = [e for e in ("allgather", "halo", "chunked", "fused") if e != args.exchange]
            for other in others:
                r2 = measure_sharded(args.workload, args.mode, args.steps, args.warmup, dev, rank, P, group,
                                     other, 0, one_gpu)
                secondary[f"exchange_{other}"] = {
                    "value": r2["value"], "unit": UNIT, "ms_per_step": r2["ms_per_step"],
                    "breakdown_ms_max_over_ranks": r2["breakdown_ms_max_over_ranks"],
                    "exchange": r2["exchange"], "roofline": r2["roofline"], "clocks": r2["clocks"]}
        m, n, nnz = res["m"], res["n"], res["nnz"]
    else:
        t0 = time.perf_counter()
        A, m, n, _ = build_local(args.workload, 0, 1)
        nnz = A.nnz
        x_h = gen.dense_x(n, 101)
        log(f"{args.workload}: {A.m}x{A.n} nnz {A.nnz} generated in {time.perf_counter() - t0:.1f}s")
        res = measure_workload(A, x_h, args.mode, args.steps, args.warmup, dev, use_graph=not args.no_graph,
                               single=True, e2e_steps=args.e2e_steps)
        # the same kernel over a long back-to-back run (a sustained solver's
        # regime: clocks settle under the power cap)
        if not args.no_secondary:
            rs = measure_workload(A, x_h, args.mode, max(300, args.steps), args.warmup, dev,
                                  use_graph=not args.no_graph, single=False, check=False)
            res["sustained"] = {"steps": max(300, args.steps), "ms_per_step": rs["ms_per_step"],
                                "frac": rs["roofline"]["frac"], "clocks": rs["clocks"]}
        if rank == 0 and not args.no_cpu_baseline:
            res["cpu_baseline"] = oracle_f64_baseline(A, x_h)
            res["cpu_context"] = cpu_context(A, x_h, res["info"], res["create_s"])
        del A
        if not args.no_secondary:
            cache = {}
            for wl, md in SECONDARY:
                if wl == args.workload and md == args.mode:
                    continue
                if wl not in cache:
                    cache.clear()
                    cache[wl] = gen.make(wl)
                B, xb = cache[wl]
                r2 = measure_workload(B, xb, md, max(args.steps, 200), args.warmup, dev,
                                      use_graph=not args.no_graph, single=True)
                secondary[f"{wl}/{md}"] = secondary_entry(r2, wl, md)
                log(f"secondary {wl}/{md}: {r2['ms_per_step'] * 1e3:.1f} us, frac {r2['roofline']['frac']:.3f}")
    if rank == 0:
        info = res["info"]
        out = {"metric": METRIC, "value": res["value"], "unit": UNIT, "n_gpus": P,
               "steps": args.steps, "warmup": args.warmup, "ms_per_step": res["ms_per_step"],
               "higher_is_better": True, "scaling": "strong" if P > 1 else "weak",
               "vs_baseline": None, "dtype": "f64", "data": "synthetic",
               "config": run_config(args, m, n, nnz, P),
               "roofline": res["roofline"],
               "cpu_baseline": res.get("cpu_baseline"),
               "e2e": res.get("e2e"),
               "gpu_launches": args.steps * res.get("launches_per_step", 1),
               "clocks": res["clocks"],
               "step": ({"allgather": "SpMV + NCCL all-gather of y",
                         "halo": "halo exchange overlapped with the interior SpMV + boundary SpMVs",
                         "chunked": f"{CHUNKS} chunk SpMVs, each chunk sent to every peer while the next "
                                    "computes",
                         "fused": "SpMV storing y into every rank's x_{k+1} (scatter epilogue) + barrier"}[args.exchange]
                        if P > 1 else "one SpMV launch"),
               "timing": {"launch_mode": res["launch_mode"], "replicas_rotated": res["reps"],
                          "host_enqueue_us_per_step": res.get("host_enqueue_us_per_step")},
               "tiling": {"numtile": info["numtile"], "rem_nnz": info["rem_nnz"],
                          "kept_tiles": dict(zip(["CSR", "COO", "ELL", "HYB", "DNS", "DNSROW", "DNSCOL"],
                                                 info["kept_tiles"])),
                          "alg_bytes_per_spmv": info["alg_bytes"], "device_bytes": info["device_bytes"],
                          "create_s": res["create_s"], "kernel": info["kernel"]},
               "launch": res["launch"],
               "parity": res.get("parity")}
        for k in ("single_launch", "sustained", "cpu_context", "exchange", "breakdown_ms_max_over_ranks"):
            if res.get(k) is not None:
                out[k] = res[k]
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
    ap.add_argument("--mode", default="DEFERRED", choices=["ADPT", "DEFERRED", "AUTO", "FORCE_CSR", "BYTES"])
    ap.add_argument("--exchange", default="allgather", choices=["allgather", "halo", "chunked", "fused"],
                    help="N>1: all-gather of y (north star, default), the neighbour-only x exchange, the all-gather in "
                         "chunks overlapped with the SpMV, or the fused scatter epilogue (no collective); "
                         "the others are timed as secondary entries")
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
