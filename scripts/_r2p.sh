cd $GRAFT_REPO_ROOT
OUT=gpurun_out/r2p; mkdir -p $OUT
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider > $OUT/tests_gpu.log 2>&1; echo rc=$? >> $OUT/tests_gpu.log
bash scripts/gpu_ab.sh r2p "fem:DEFERRED fem:BYTES stencil27_200:BYTES mixed:BYTES rmat20:BYTES mixed:ADPT" bytes
