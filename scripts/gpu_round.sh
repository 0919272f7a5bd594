#!/bin/bash
# Full GPU evidence pass: smoke, GPU tests, the driver's bench command, the
# ncu launch list of that command, one ncu --set full capture per config,
# compute-sanitizer over small matrices.  usage: scripts/gpu_round.sh TAG
cd $GRAFT_REPO_ROOT
TAG=${1:-r2}
OUT=gpurun_out/$TAG
mkdir -p $OUT
NCU=/usr/local/cuda/bin/ncu
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > $OUT/gpu.txt 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.log 2>&1; echo "rc=$?" >> $OUT/smoke.log
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider > $OUT/tests_gpu.log 2>&1; echo "rc=$?" >> $OUT/tests_gpu.log
timeout 900 python bench.py --gpus 1 --steps 20 --warmup 5 > $OUT/bench_default.json 2> $OUT/bench_default.err; echo "rc=$?" >> $OUT/bench_default.err
timeout 900 $NCU --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches.csv \
   python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-secondary --e2e-steps 1 > $OUT/launches_bench.log 2>&1
for wm in stencil27_200:DEFERRED fem:DEFERRED rmat20:DEFERRED mixed:ADPT mixed:DEFERRED; do
  w=${wm%%:*}; m=${wm#*:}
  timeout 900 $NCU --set full --clock-control none --import-source on -k regex:tilespmv_fp64 -s 3 -c 1 \
     -o $OUT/full_${w}_${m} -f python bench.py --workload $w --mode $m --steps 2 --warmup 3 --no-cpu-baseline \
     --no-secondary --e2e-steps 0 > $OUT/full_${w}_${m}.log 2>&1
done
# (compute-sanitizer is closed on the GPU pool since round 2; the r02_v2
# sanitizer logs are the last ones)
# the N > 1 code path on one GPU (two ranks on cuda:0 over gloo, host-staged exchange): a functional
# check of bench.py's sharded step, not a bench number
TILESPMV_BENCH_ONE_GPU=1 timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 \
   --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --steps 5 --warmup 3 --workload stencil27_40 \
   --e2e-steps 2 > $OUT/n2_devcheck.json 2> $OUT/n2_devcheck.err; echo "rc=$?" >> $OUT/n2_devcheck.err
timeout 300 python bench.py --impl reference --steps 20 --warmup 5 > $OUT/reference.json 2> $OUT/reference.err
timeout 800 python scripts/checked_small.py > $OUT/checked_small.log 2>&1; echo "rc=$?" >> $OUT/checked_small.log
timeout 1200 python scripts/paper_ablation.py > $OUT/ablation.jsonl 2> $OUT/ablation.err
timeout 600 python scripts/cg_bench.py > $OUT/cg_stencil27_200.json 2> $OUT/cg.err
echo done > $OUT/DONE
