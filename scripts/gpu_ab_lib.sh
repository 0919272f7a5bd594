#!/bin/bash
# A/B of two builds of libtilespmv.so on one box: copy the baseline build to
# ab_old/libtilespmv.so (git-ignored, travels with gpurun), rebuild the
# candidate in place, then run this; interleaved bench lines -> summary.txt.
cd $GRAFT_REPO_ROOT
OUT=gpurun_out/flatpair; mkdir -p $OUT
PKG=paper_conf_ipps_niuldj0t21_b200
cp $PKG/libtilespmv.so ab_old/new.so
timeout 600 python -m pytest tests -m gpu -q > $OUT/tests_gpu.log 2>&1; echo rc=$? >> $OUT/tests_gpu.log
timeout 120 python scripts/sanitize_small.py > $OUT/sanity.log 2>&1; echo rc=$? >> $OUT/sanity.log
for r in 1 2; do
 for v in new old; do
  if [ $v = new ]; then cp ab_old/new.so $PKG/libtilespmv.so; else cp ab_old/libtilespmv.so $PKG/libtilespmv.so; fi
  touch $PKG/libtilespmv.so
  for wl in rmat20 mixed:ADPT mixed stencil27_200; do
    w=${wl%%:*}; m=DEFERRED; [ "$wl" != "$w" ] && m=${wl#*:}
    timeout 300 python bench.py --workload $w --mode $m --steps 200 --no-secondary --no-cpu-baseline --e2e-steps 2 > $OUT/b_${v}_${r}_${w}_${m}.json 2>/dev/null
  done
 done
done
cp ab_old/new.so $PKG/libtilespmv.so; touch $PKG/libtilespmv.so
python - > $OUT/summary.txt <<'PY'
import json,glob
for f in sorted(glob.glob("gpurun_out/flatpair/b_*.json")):
    try:
        d=json.loads(open(f).read().strip().splitlines()[-1]); print(f.split('/')[-1], round(d["ms_per_step"]*1000,1), "us", round(d["roofline"]["frac"],3), d["clocks"]["sm_mhz"])
    except Exception as e: print(f, "ERR", e)
PY
