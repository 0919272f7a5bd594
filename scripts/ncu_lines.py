#!/usr/bin/env python
"""Per-source-line instruction and stall-sample totals of an ncu report
(--import-source on, -lineinfo build):

    python scripts/ncu_lines.py REPORT.ncu-rep [--top N]
"""
import csv
import io
import subprocess
import sys

NCU = "/usr/local/cuda/bin/ncu"


def main():
    rep = sys.argv[1]
    top = int(sys.argv[sys.argv.index("--top") + 1]) if "--top" in sys.argv else 40
    out = subprocess.run([NCU, "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                         capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    fname, hdr, agg = "", None, {}
    cur = None
    for r in rows:
        if len(r) == 2 and r[0] == "File Path":
            fname = r[1].split("/")[-1]
            continue
        if r and r[0] == "Line No":
            hdr = r
            continue
        if hdr is None or len(r) < len(hdr):
            continue
        if r[0]:  # a source line row
            cur = (fname, int(r[0]), r[1].strip()[:80])
            continue
        if cur is None:
            continue
        d = agg.setdefault(cur, [0, 0])
        try:
            d[0] += int(r[hdr.index("Warp Stall Sampling (All Samples)")])
            d[1] += int(r[hdr.index("Instructions Executed")])
        except ValueError:
            pass
    ts = sum(v[0] for v in agg.values()) or 1
    ti = sum(v[1] for v in agg.values()) or 1
    print(f"total stall samples {ts}, warp instructions {ti}")
    print("| stall % | inst % | file:line | source |")
    print("|---|---|---|---|")
    for k, v in sorted(agg.items(), key=lambda kv: -kv[1][0])[:top]:
        print(f"| {100 * v[0] / ts:5.1f} | {100 * v[1] / ti:5.1f} | {k[0]}:{k[1]} | `{k[2]}` |")


if __name__ == "__main__":
    main()
