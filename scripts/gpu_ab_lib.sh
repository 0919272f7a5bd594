#!/bin/bash
# A/B of two builds of libtilespmv.so on one box: copy the baseline build to
# ab_old/libtilespmv.so (git-ignored, travels with gpurun), rebuild the
# candidate in place, then run this; interleaved bench lines -> summary.txt.
cd $GRAFT_REPO_ROOT
OUT=gpurun_out/${1:-ab}; mkdir -p $OUT
PKG=paper_conf_ipps_niuldj0t21_b200
cp $PKG/libtilespmv.so ab_old/new.so
timeout 600 python -m pytest tests -m gpu -q > $OUT/tests_gpu.log 2>&1; echo rc=$? >> $OUT/tests_gpu.log
timeout 120 python scripts/sanitize_small.py > $OUT/sanity.log 2>&1; echo rc=$? >> $OUT/sanity.log
python scripts/ab_dump_y.py $OUT/y_new.npz
cp ab_old/libtilespmv.so $PKG/libtilespmv.so; touch $PKG/libtilespmv.so; python scripts/ab_dump_y.py $OUT/y_old.npz
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
python -c "import numpy as np,sys; a=np.load(sys.argv[1]); b=np.load(sys.argv[2]); print({k: bool(np.array_equal(a[k].view(np.uint64), b[k].view(np.uint64))) for k in a.files})" $OUT/y_new.npz $OUT/y_old.npz > $OUT/bitwise.txt 2>&1; rm -f $OUT/y_*.npz
python - $OUT > $OUT/summary.txt <<'PY'
import json,glob,sys
for f in sorted(glob.glob(sys.argv[1] + "/b_*.json")):
    try:
        d=json.loads(open(f).read().strip().splitlines()[-1]); print(f.split('/')[-1], round(d["ms_per_step"]*1000,1), "us", round(d["roofline"]["frac"],3), d["clocks"]["sm_mhz"])
    except Exception as e: print(f, "ERR", e)
PY
