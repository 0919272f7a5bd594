cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/r2h
timeout 1200 python -m pytest tests -m gpu -q -x -p no:cacheprovider > gpurun_out/r2h/tests_gpu.log 2>&1; echo rc=$? >> gpurun_out/r2h/tests_gpu.log
bash scripts/gpu_ab.sh r2h "rmat20:DEFERRED mixed:DEFERRED mixed:ADPT stencil27_200:DEFERRED fem:DEFERRED" gk r01_head
