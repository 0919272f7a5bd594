cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/r2b
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider -x > gpurun_out/r2b/tests_gpu.log 2>&1; echo "rc=$?" >> gpurun_out/r2b/tests_gpu.log
bash scripts/gpu_ab.sh r2b "rmat20:DEFERRED mixed:DEFERRED mixed:ADPT stencil27_200:DEFERRED fem:DEFERRED lap2d_64:DEFERRED" d3 d4 r01_head
