cd $GRAFT_REPO_ROOT
OUT=gpurun_out/r2n; mkdir -p $OUT
timeout 1200 python -m pytest tests -m gpu -q -x -p no:cacheprovider > $OUT/tests_gpu.log 2>&1; echo rc=$? >> $OUT/tests_gpu.log
bash scripts/gpu_ab.sh r2n "mixed:ADPT rmat20:ADPT stencil27_200:ADPT mixed:DEFERRED" run norun
