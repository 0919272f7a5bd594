#!/bin/bash
# ncu --set full of the SpMV kernel on the weaker configs + the paper-figure ablation.
# usage: scripts/gpu_profile_more.sh TAG
cd $GRAFT_REPO_ROOT
TAG=${1:-r1}
OUT=gpurun_out/$TAG
mkdir -p $OUT
NCU=/usr/local/cuda/bin/ncu
for spec in "rmat20 DEFERRED" "mixed DEFERRED" "mixed ADPT"; do
  set -- $spec
  timeout 900 $NCU --set full --clock-control none --import-source on -k regex:tilespmv_fp64 -s 3 -c 1 \
     -o $OUT/full_$1_$2 -f python bench.py --workload $1 --mode $2 --steps 2 --warmup 3 --no-cpu-baseline \
     --no-secondary --e2e-steps 1 > $OUT/full_$1_$2.log 2>&1
done
timeout 1500 python scripts/paper_ablation.py > $OUT/ablation.jsonl 2> $OUT/ablation.err
echo done > $OUT/DONE
