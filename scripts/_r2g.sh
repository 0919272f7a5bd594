cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/r2g
timeout 600 python scripts/microbench/gather_bench.py rmat20 > gpurun_out/r2g/gather_rmat20_smem.txt 2>&1
