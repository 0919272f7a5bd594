#!/bin/bash
# ncu --set full of one SpMV launch: scripts/ncu_one.sh TAG WORKLOAD MODE [extra env]
cd $GRAFT_REPO_ROOT
TAG=$1; WL=$2; MODE=${3:-DEFERRED}
OUT=gpurun_out/$TAG
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 900 /usr/local/cuda/bin/ncu --set full --clock-control none --import-source on -k regex:tilespmv_fp64 -s 3 -c 1 \
   -o $OUT/full_${WL}_${MODE} -f python bench.py --workload $WL --mode $MODE --steps 2 --warmup 3 --no-cpu-baseline \
   --no-secondary --e2e-steps 1 > $OUT/full_${WL}_${MODE}.log 2>&1
echo done > $OUT/DONE
