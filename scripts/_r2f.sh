cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/r2f
timeout 600 python scripts/microbench/gather_bench.py rmat20 > gpurun_out/r2f/gather_rmat20.txt 2>&1
