cd $GRAFT_REPO_ROOT
OUT=gpurun_out/r2u; mkdir -p $OUT
timeout 600 python scripts/ab_bench.py rmat20 GATHER,24,25,26,27 --rounds 5 --steps 100 > $OUT/ab_rmat20.txt 2>&1
