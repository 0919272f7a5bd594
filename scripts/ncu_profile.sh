#!/bin/bash
# usage: scripts/ncu_profile.sh TAG WORKLOAD MODE
# Writes gpurun_out/TAG_launches.csv (every launch, gpu__time_duration) and
# gpurun_out/TAG_full.ncu-rep (ncu --set full of one SpMV launch).
cd $GRAFT_REPO_ROOT
TAG=$1; WL=${2:-stencil27_200}; MODE=${3:-DEFERRED}
NCU=/usr/local/cuda/bin/ncu
timeout 900 $NCU --metrics gpu__time_duration.sum --clock-control none --csv \
   --log-file gpurun_out/${TAG}_launches.csv \
   python bench.py --workload $WL --mode $MODE --steps 5 --warmup 3 --no-cpu-baseline --no-secondary --e2e-steps 1 \
   > gpurun_out/${TAG}_launches_bench.log 2>&1
timeout 1200 $NCU --set full --clock-control none --import-source on -k regex:tilespmv_fp64 -s 3 -c 1 \
   -o gpurun_out/${TAG}_full -f \
   python bench.py --workload $WL --mode $MODE --steps 2 --warmup 3 --no-cpu-baseline --no-secondary --e2e-steps 1 \
   > gpurun_out/${TAG}_full_bench.log 2>&1
echo "ncu done rc=$?" >> gpurun_out/${TAG}_full_bench.log
