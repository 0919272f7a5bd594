cd $GRAFT_REPO_ROOT
PKG=paper_conf_ipps_niuldj0t21_b200
cp ab_old/g.so $PKG/libtilespmv.so; touch $PKG/libtilespmv.so
mkdir -p gpurun_out/r2e
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fuzz.py -m gpu -q -x -p no:cacheprovider > gpurun_out/r2e/tests_g.log 2>&1; echo rc=$? >> gpurun_out/r2e/tests_g.log
bash scripts/gpu_ab.sh r2e "rmat20:DEFERRED mixed:DEFERRED stencil27_200:DEFERRED" g g_med d3 r01_head
