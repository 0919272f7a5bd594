cd $GRAFT_REPO_ROOT
OUT=gpurun_out/r2i; mkdir -p $OUT
timeout 900 /usr/local/cuda/bin/ncu --set full --clock-control none --import-source on -k regex:tilespmv_fp64 -s 3 -c 1 \
      -o $OUT/full_gk_rmat20 -f python bench.py --workload rmat20 --steps 2 --warmup 3 --no-cpu-baseline \
      --no-secondary --e2e-steps 0 > $OUT/full_gk_rmat20.log 2>&1
