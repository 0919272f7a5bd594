#!/bin/bash
# Round-2 GPU pass: smoke, GPU tests, the driver's bench command, and an
# old-vs-new A/B of short bench lines (ab_old/r01_head.so = round-1 HEAD).
# usage: scripts/gpu_r2.sh TAG [no-ab]
cd $GRAFT_REPO_ROOT
TAG=${1:-r2}
OUT=gpurun_out/$TAG
mkdir -p $OUT
PKG=paper_conf_ipps_niuldj0t21_b200
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > $OUT/gpu.txt 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.log 2>&1; echo "rc=$?" >> $OUT/smoke.log
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider > $OUT/tests_gpu.log 2>&1; echo "rc=$?" >> $OUT/tests_gpu.log
timeout 900 python bench.py --gpus 1 --steps 20 --warmup 5 > $OUT/bench_default.json 2> $OUT/bench_default.err; echo "rc=$?" >> $OUT/bench_default.err
if [ "$2" != "no-ab" ] && [ -f ab_old/r01_head.so ]; then
  cp $PKG/libtilespmv.so ab_old/new.so
  for r in 1 2; do
    for v in new old; do
      if [ $v = new ]; then cp ab_old/new.so $PKG/libtilespmv.so; else cp ab_old/r01_head.so $PKG/libtilespmv.so; fi
      touch $PKG/libtilespmv.so
      for wl in rmat20:DEFERRED mixed:ADPT mixed:DEFERRED stencil27_200:DEFERRED fem:DEFERRED; do
        w=${wl%%:*}; m=${wl#*:}
        timeout 300 python bench.py --workload $w --mode $m --steps 200 --no-secondary --no-cpu-baseline --e2e-steps 0 > $OUT/ab_${v}_${r}_${w}_${m}.json 2>/dev/null
      done
    done
  done
  cp ab_old/new.so $PKG/libtilespmv.so; touch $PKG/libtilespmv.so
  python - $OUT > $OUT/ab_summary.txt <<'PY'
import json,glob,sys
for f in sorted(glob.glob(sys.argv[1] + "/ab_*.json")):
    try:
        d=json.loads(open(f).read().strip().splitlines()[-1]); s=d.get("single_launch",{})
        print(f.split('/')[-1], round(d["ms_per_step"]*1000,1), "us", round(d["roofline"]["frac"],3), "single", round(s.get("median_ms",0)*1000,1), d["clocks"]["sm_mhz"], d["clocks"]["reasons"])
    except Exception as e: print(f, "ERR", e)
PY
fi
echo done > $OUT/DONE
