#!/bin/bash
# Full GPU pass: tests, default bench line, per-workload lines, ncu evidence.
# usage: scripts/gpu_round.sh TAG
cd $GRAFT_REPO_ROOT
TAG=${1:-r1}
OUT=gpurun_out/$TAG
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.log 2>&1; echo "rc=$?" >> $OUT/smoke.log
timeout 1500 python -m pytest tests -m gpu -q > $OUT/tests_gpu.log 2>&1; echo "rc=$?" >> $OUT/tests_gpu.log
timeout 900 python bench.py > $OUT/bench_default.json 2> $OUT/bench_default.err; echo "rc=$?" >> $OUT/bench_default.err
for wl in fem mixed rmat20 lap2d_64; do
  timeout 600 python bench.py --workload $wl --no-secondary --cpu-seconds 3 --e2e-steps 5 > $OUT/bench_$wl.json 2> $OUT/bench_$wl.err
done
timeout 600 python bench.py --workload mixed --mode ADPT --no-secondary --cpu-seconds 3 --e2e-steps 5 > $OUT/bench_mixed_adpt.json 2> $OUT/bench_mixed_adpt.err
NCU=/usr/local/cuda/bin/ncu
timeout 900 $NCU --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches.csv \
   python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-secondary --e2e-steps 1 > $OUT/launches_bench.log 2>&1
timeout 1200 $NCU --set full --clock-control none --import-source on -k regex:tilespmv_fp64 -s 3 -c 1 \
   -o $OUT/full_stencil -f python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-secondary --e2e-steps 1 > $OUT/full_stencil.log 2>&1
timeout 900 $NCU --set full --clock-control none --import-source on -k regex:tilespmv_fp64 -s 3 -c 1 \
   -o $OUT/full_fem -f python bench.py --workload fem --steps 2 --warmup 3 --no-cpu-baseline --no-secondary --e2e-steps 1 > $OUT/full_fem.log 2>&1
for tool in memcheck racecheck synccheck initcheck; do
  timeout 900 /usr/local/cuda/bin/compute-sanitizer --tool $tool --num-cuda-barriers 64 --error-exitcode 9 python scripts/sanitize_small.py > $OUT/sanitizer_$tool.log 2>&1
  echo "rc=$?" >> $OUT/sanitizer_$tool.log
done
echo done > $OUT/DONE
