cd $GRAFT_REPO_ROOT
OUT=gpurun_out/r2o; mkdir -p $OUT
timeout 600 python scripts/ab_bench.py rmat20 GATHER,20,21 --rounds 3 --steps 50 > $OUT/ab_rmat20.txt 2>&1
