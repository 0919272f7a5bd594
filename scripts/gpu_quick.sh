#!/bin/bash
# Quick GPU check after a kernel change: GPU tests, then one short bench line
# per workload (no CPU baseline).  usage: scripts/gpu_quick.sh TAG [workloads...]
cd $GRAFT_REPO_ROOT
TAG=${1:-quick}; shift
WLS=${@:-"stencil27_200 fem rmat20 mixed"}
OUT=gpurun_out/$TAG
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 900 python -m pytest tests -m gpu -x -q > $OUT/tests_gpu.log 2>&1; echo "rc=$?" >> $OUT/tests_gpu.log
for wl in $WLS; do
  timeout 300 python bench.py --workload $wl --steps 200 --no-secondary --no-cpu-baseline --e2e-steps 3 > $OUT/bench_$wl.json 2> $OUT/bench_$wl.err
done
timeout 300 python bench.py --workload mixed --mode ADPT --steps 200 --no-secondary --no-cpu-baseline --e2e-steps 3 > $OUT/bench_mixed_adpt.json 2> $OUT/bench_mixed_adpt.err
echo done > $OUT/DONE
