cd $GRAFT_REPO_ROOT
OUT=gpurun_out/r2t; mkdir -p $OUT
timeout 600 python scripts/ab_bench.py stencil27_200 SM_QUEUE,22 --rounds 7 --steps 100 > $OUT/ab_c5.txt 2>&1
timeout 600 python scripts/ab_bench.py mixed SM_QUEUE,22 --rounds 5 --steps 100 > $OUT/ab_mixed.txt 2>&1
timeout 600 python scripts/ab_bench.py mixed SM_QUEUE,22 --mode ADPT --rounds 5 --steps 100 > $OUT/ab_mixed_adpt.txt 2>&1
timeout 600 python scripts/ab_bench.py rmat20 GATHER,23 --rounds 5 --steps 100 > $OUT/ab_rmat20.txt 2>&1
