#!/bin/bash
# A/B of kernel variants plus an ncu capture (with per-SASS source counters)
# of one variant on the stencil: scripts/gpu_ab.sh TAG VARIANTS NCU_VARIANT [WORKLOADS]
cd $GRAFT_REPO_ROOT
TAG=$1; VARS=$2; NV=$3; WLS=${4:-"stencil27_200 mixed rmat20"}
OUT=gpurun_out/$TAG
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 600 python -m pytest tests -m gpu -x -q -k "variants_parity or row_slices or pool" > $OUT/tests_gpu.log 2>&1; echo "rc=$?" >> $OUT/tests_gpu.log
for wl in $WLS; do
  timeout 300 python scripts/ab_bench.py $wl $VARS > $OUT/ab_$wl.txt 2>&1
done
timeout 300 python scripts/ab_bench.py mixed $VARS --mode ADPT > $OUT/ab_mixed_adpt.txt 2>&1
if [ -n "$NV" ]; then
  TILESPMV_KERNEL=$NV timeout 900 /usr/local/cuda/bin/ncu --set full --clock-control none --import-source on -k regex:tilespmv_fp64 -s 3 -c 1 \
     -o $OUT/full_stencil -f python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-secondary --e2e-steps 1 > $OUT/full_stencil.log 2>&1
  /usr/local/cuda/bin/ncu -i $OUT/full_stencil.ncu-rep --page source --csv --print-source sass > $OUT/source_stencil.csv 2>&1
fi
echo done > $OUT/DONE
