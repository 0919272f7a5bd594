cd $GRAFT_REPO_ROOT
OUT=gpurun_out/r2k; mkdir -p $OUT
timeout 600 python scripts/ab_bench.py rmat20 SM_QUEUE,GATHER,14,15 --rounds 3 --steps 50 > $OUT/ab_rmat20.txt 2>&1
bash scripts/gpu_ab.sh r2k "rmat20:DEFERRED mixed:DEFERRED mixed:ADPT stencil27_200:DEFERRED" rb r01_head
