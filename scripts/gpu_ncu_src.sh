#!/bin/bash
# ncu --set full (+ per-SASS source counters) of the default kernel on
# several workload[:mode] specs: scripts/gpu_ncu_src.sh TAG SPEC...
cd $GRAFT_REPO_ROOT
TAG=$1; shift
OUT=gpurun_out/$TAG
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
for spec in "$@"; do
  WL=${spec%%:*}; MODE=DEFERRED; [ "$spec" != "$WL" ] && MODE=${spec#*:}
  timeout 900 /usr/local/cuda/bin/ncu --set full --clock-control none --import-source on -k regex:tilespmv_fp64 -s 3 -c 1 \
     -o $OUT/full_${WL}_${MODE} -f python bench.py --workload $WL --mode $MODE --steps 2 --warmup 3 --no-cpu-baseline \
     --no-secondary --e2e-steps 1 > $OUT/full_${WL}_${MODE}.log 2>&1
  /usr/local/cuda/bin/ncu -i $OUT/full_${WL}_${MODE}.ncu-rep --page source --csv --print-source sass > $OUT/source_${WL}_${MODE}.csv 2>&1
done
echo done > $OUT/DONE
