cd $GRAFT_REPO_ROOT
OUT=gpurun_out/r2j; mkdir -p $OUT
timeout 600 python scripts/ab_bench.py rmat20 SM_QUEUE,GATHER,10,11,12,13,14 --rounds 3 --steps 50 > $OUT/ab_rmat20.txt 2>&1
