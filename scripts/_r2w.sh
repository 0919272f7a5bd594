cd $GRAFT_REPO_ROOT
OUT=gpurun_out/r2w; mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "kernels_parity or row_slices or full_size" -p no:cacheprovider > $OUT/tests_gpu.log 2>&1; echo rc=$? >> $OUT/tests_gpu.log
timeout 600 python scripts/ab_bench.py rmat20 GATHER,28 --rounds 5 --steps 100 > $OUT/ab_rmat20.txt 2>&1
timeout 600 python scripts/ab_bench.py stencil27_200 SM_QUEUE,29 --rounds 5 --steps 100 > $OUT/ab_c5.txt 2>&1
timeout 600 python scripts/ab_bench.py mixed SM_QUEUE,29 --rounds 5 --steps 100 > $OUT/ab_mixed.txt 2>&1
timeout 600 python scripts/ab_bench.py mixed SM_QUEUE,29 --mode ADPT --rounds 5 --steps 100 > $OUT/ab_mixed_adpt.txt 2>&1
