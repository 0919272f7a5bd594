#!/bin/bash
# GPU tests + A/B + ncu (source counters) of the default kernel on one workload:
# scripts/gpu_ab2.sh TAG VARIANTS NCU_WORKLOAD [WORKLOADS]
cd $GRAFT_REPO_ROOT
TAG=$1; VARS=$2; NW=$3; WLS=${4:-"stencil27_200 mixed rmat20"}
OUT=gpurun_out/$TAG
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 120 python scripts/sanitize_small.py > $OUT/sanity.log 2>&1 || { echo sanity-fail > $OUT/DONE; exit 1; }
timeout 600 python -m pytest tests -m gpu -x -q > $OUT/tests_gpu.log 2>&1; echo "rc=$?" >> $OUT/tests_gpu.log
for wl in $WLS; do
  timeout 240 python scripts/ab_bench.py $wl $VARS > $OUT/ab_$wl.txt 2>&1
done
if [ -n "$NW" ]; then
  timeout 900 /usr/local/cuda/bin/ncu --set full --clock-control none --import-source on -k regex:tilespmv_fp64 -s 3 -c 1 \
     -o $OUT/full_$NW -f python bench.py --workload $NW --steps 2 --warmup 3 --no-cpu-baseline --no-secondary --e2e-steps 1 > $OUT/full_$NW.log 2>&1
  /usr/local/cuda/bin/ncu -i $OUT/full_$NW.ncu-rep --page source --csv --print-source sass > $OUT/source_$NW.csv 2>&1
fi
echo done > $OUT/DONE
