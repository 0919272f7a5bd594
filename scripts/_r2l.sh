cd $GRAFT_REPO_ROOT
OUT=gpurun_out/r2l; mkdir -p $OUT
timeout 1200 python -m pytest tests -m gpu -q -x -p no:cacheprovider > $OUT/tests_gpu.log 2>&1; echo rc=$? >> $OUT/tests_gpu.log
timeout 600 python scripts/ab_bench.py rmat20 SM_QUEUE,GATHER,14,15,16 --rounds 3 --steps 50 > $OUT/ab_rmat20.txt 2>&1
timeout 600 python scripts/ab_bench.py stencil27_200 SM_QUEUE --rounds 5 --steps 100 > $OUT/ab_c5.txt 2>&1
cp ab_old/r01_head.so paper_conf_ipps_niuldj0t21_b200/libtilespmv.so; touch paper_conf_ipps_niuldj0t21_b200/libtilespmv.so
timeout 600 python scripts/ab_bench.py stencil27_200 AUTO --rounds 5 --steps 100 > $OUT/ab_c5_r01.txt 2>&1
cp ab_old/rc.so paper_conf_ipps_niuldj0t21_b200/libtilespmv.so; touch paper_conf_ipps_niuldj0t21_b200/libtilespmv.so
timeout 900 /usr/local/cuda/bin/ncu --set full --clock-control none --import-source on -k regex:tilespmv_fp64 -s 3 -c 1 \
      -o $OUT/full_rmat20 -f python bench.py --workload rmat20 --steps 2 --warmup 3 --no-cpu-baseline \
      --no-secondary --e2e-steps 0 > $OUT/full_rmat20.log 2>&1
