#!/usr/bin/env python
"""Summarise an `ncu --set full` report of the SpMV kernel for profiles/.

    python scripts/ncu_summary.py gpurun_out/TAG_full.ncu-rep [--alg-bytes B] [--key WL/MODE]

Prints a markdown summary (duration, DRAM bytes, throughput, L2 hit rate,
occupancy, issue activity, warp-stall breakdown, hottest SASS) and, with
--key, records the per-launch DRAM traffic in profiles/ncu_traffic.json (the
`traffic` field of bench.py's roofline object).
"""
import argparse
import csv
import io
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
NCU = "/usr/local/cuda/bin/ncu"

METRICS = [
    ("gpu__time_duration.sum", "duration"),
    ("dram__bytes_read.sum", "DRAM read"),
    ("dram__bytes_write.sum", "DRAM write"),
    ("dram__throughput.avg.pct_of_peak_sustained_elapsed", "DRAM throughput % of peak"),
    ("lts__throughput.avg.pct_of_peak_sustained_elapsed", "L2 throughput % of peak"),
    ("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "GPU DRAM throughput %"),
    ("lts__t_sector_hit_rate.pct", "L2 sector hit rate"),
    ("lts__t_bytes.sum", "L2 bytes"),
    ("l1tex__t_sector_hit_rate.pct", "L1 sector hit rate"),
    ("sm__warps_active.avg.pct_of_peak_sustained_active", "warps active % (occupancy)"),
    ("smsp__issue_active.avg.pct_of_peak_sustained_active", "issue active %"),
    ("smsp__inst_executed.sum", "warp instructions"),
    ("sm__throughput.avg.pct_of_peak_sustained_elapsed", "SM throughput %"),
    ("launch__registers_per_thread", "registers/thread"),
    ("launch__grid_size", "grid"),
    ("launch__block_size", "block"),
    ("launch__shared_mem_per_block_dynamic", "dynamic smem/CTA"),
]


def raw(rep):
    out = subprocess.run([NCU, "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units = rows[0], rows[1]
    launches = []
    for r in rows[2:]:
        launches.append({h: (v, u) for h, u, v in zip(hdr, units, r)})
    return launches


def to_bytes(v, u):
    f = float(v.replace(",", ""))
    return f * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}.get(u, 1)


def sass_top(rep, n=25):
    out = subprocess.run([NCU, "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                         capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hi = next(i for i, r in enumerate(rows) if "Source" in r and "Instructions Executed" in r)
    hdr = rows[hi]
    ie, iss, isrc = hdr.index("Instructions Executed"), hdr.index("Warp Stall Sampling (All Samples)"), hdr.index("Source")
    data = [r for r in rows[hi + 1:] if len(r) > ie]
    tot = sum(float(r[ie] or 0) for r in data) or 1
    stot = sum(float(r[iss] or 0) for r in data) or 1
    data.sort(key=lambda r: -float(r[iss] or 0))
    lines = [f"| {float(r[iss] or 0) / stot * 100:5.1f}% | {float(r[ie] or 0) / tot * 100:5.2f}% | `{r[isrc].strip()[:70]}` |"
             for r in data[:n]]
    return lines


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("rep")
    ap.add_argument("--alg-bytes", type=float, default=None)
    ap.add_argument("--key", default=None)
    ap.add_argument("--title", default="")
    a = ap.parse_args()
    L = raw(a.rep)
    for i, d in enumerate(L):
        name = d.get("Kernel Name", ("?", ""))[0]
        print(f"## {a.title} launch {i}: `{name[:110]}`\n")
        print("| metric | value |\n|---|---|")
        for k, label in METRICS:
            if k in d:
                v, u = d[k]
                print(f"| {label} (`{k}`) | {v} {u} |")
        stalls = sorted(((k, float(v[0].replace(',', '') or 0)) for k, v in d.items()
                         if k.startswith("smsp__average_warps_issue_stalled_") and k.endswith("_per_issue_active.ratio")),
                        key=lambda t: -t[1])
        if stalls:
            print("\nwarp stall reasons (cycles per issued instruction):\n")
            for k, v in stalls[:8]:
                print(f"- {k.replace('smsp__average_warps_issue_stalled_', '').replace('_per_issue_active.ratio', '')}: {v:.2f}")
        try:
            rd = to_bytes(*d["dram__bytes_read.sum"])
            wr = to_bytes(*d["dram__bytes_write.sum"])
            dur = float(d["gpu__time_duration.sum"][0].replace(",", ""))
            unit = d["gpu__time_duration.sum"][1]
            sec = dur * {"nsecond": 1e-9, "usecond": 1e-6, "msecond": 1e-3, "second": 1,
                         "ns": 1e-9, "us": 1e-6, "ms": 1e-3, "s": 1}[unit]
            print(f"\nDRAM traffic per launch: {rd + wr:.4g} B ({(rd + wr) / sec / 1e9:.1f} GB/s over the ncu duration)")
            if a.alg_bytes:
                print(f"algorithmic bytes: {a.alg_bytes:.4g} B -> traffic / algorithmic = {(rd + wr) / a.alg_bytes:.3f}")
            if a.key:
                p = os.path.join(ROOT, "profiles", "ncu_traffic.json")
                j = json.load(open(p)) if os.path.exists(p) else {}
                j[a.key] = rd + wr
                json.dump(j, open(p, "w"), indent=1, sort_keys=True)
        except Exception as e:
            print("traffic: n/a", e, file=sys.stderr)
        print("\nhottest SASS by stall samples (stall share | instruction share | instruction):\n")
        print("| stall | inst | SASS |\n|---|---|---|")
        for line in sass_top(a.rep):
            print(line)
        print()


if __name__ == "__main__":
    main()
