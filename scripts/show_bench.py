#!/usr/bin/env python
"""One summary line per bench JSON file: python scripts/show_bench.py FILES..."""
import json
import sys

for f in sys.argv[1:]:
    try:
        d = json.loads(open(f).read().strip().splitlines()[-1])
        r = d["roofline"]
        print(f"{d['config']['workload']:14s} {d['config']['mode']:9s} {d['value']:8.1f} GF/s "
              f"{d['ms_per_step'] * 1e3:9.2f} us frac {r['frac']:.3f} {r['kernel']:30s} "
              f"clk {d['clocks'] and d['clocks']['sm_mhz']} {d['clocks'] and d['clocks']['reasons']}")
    except Exception as e:
        print(f, "unreadable:", e)
