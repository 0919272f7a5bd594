cd $GRAFT_REPO_ROOT
OUT=gpurun_out/r2s; mkdir -p $OUT
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_sharded.py -m gpu -q -x -p no:cacheprovider > $OUT/tests_gpu.log 2>&1; echo rc=$? >> $OUT/tests_gpu.log
bash scripts/gpu_ab.sh r2s "rmat20:DEFERRED stencil27_200:DEFERRED mixed:DEFERRED" acqrel local
