#!/bin/bash
# Interleaved A/B of library builds on one box: ab_old/<name>.so for each
# name given (git-ignored, travels with gpurun).  Short bench lines (pipelined
# + single launch) per workload, 2 rounds; summary in ab_summary.txt.
# usage: scripts/gpu_ab.sh TAG "wl:mode wl:mode ..." name1 name2 ...
cd $GRAFT_REPO_ROOT
TAG=$1; WLS=$2; shift 2
OUT=gpurun_out/$TAG
mkdir -p $OUT
PKG=paper_conf_ipps_niuldj0t21_b200
cp $PKG/libtilespmv.so $OUT/../.cur.so 2>/dev/null
for r in 1 2; do
  for v in "$@"; do
    cp ab_old/$v.so $PKG/libtilespmv.so; touch $PKG/libtilespmv.so
    for wl in $WLS; do
      w=${wl%%:*}; m=${wl#*:}
      timeout 300 python bench.py --workload $w --mode $m --steps 200 --no-secondary --no-cpu-baseline --e2e-steps 0 > $OUT/ab_${v}_${r}_${w}_${m}.json 2>/dev/null
    done
  done
done
cp $OUT/../.cur.so $PKG/libtilespmv.so; touch $PKG/libtilespmv.so
python - $OUT > $OUT/ab_summary.txt <<'PY'
import json,glob,sys
for f in sorted(glob.glob(sys.argv[1] + "/ab_*.json")):
    try:
        d=json.loads(open(f).read().strip().splitlines()[-1]); s=d.get("single_launch",{})
        s = s.get("graph", s)
        print(f.split('/')[-1], round(d["ms_per_step"]*1000,1), "us", round(d["roofline"]["frac"],3), "single", round(s.get("median_ms",0)*1000,1), d["clocks"]["sm_mhz"], d["clocks"]["reasons"])
    except Exception as e: print(f, "ERR", e)
PY
