cd $GRAFT_REPO_ROOT
OUT=gpurun_out/r2r; mkdir -p $OUT
PKG=paper_conf_ipps_niuldj0t21_b200
timeout 1500 python -m pytest tests -m gpu -q -x -p no:cacheprovider > $OUT/tests_gpu.log 2>&1; echo rc=$? >> $OUT/tests_gpu.log
python scripts/ab_dump_y.py $OUT/y_new.npz
cp ab_old/bytes.so $PKG/libtilespmv.so; touch $PKG/libtilespmv.so; python scripts/ab_dump_y.py $OUT/y_old.npz
cp ab_old/local.so $PKG/libtilespmv.so; touch $PKG/libtilespmv.so
python -c "import numpy as np,sys; a=np.load(sys.argv[1]); b=np.load(sys.argv[2]); print({k: bool(np.array_equal(a[k].view(np.uint64), b[k].view(np.uint64))) for k in a.files})" $OUT/y_new.npz $OUT/y_old.npz > $OUT/bitwise.txt 2>&1; rm -f $OUT/y_*.npz
bash scripts/gpu_ab.sh r2r "mixed:DEFERRED stencil27_200:DEFERRED rmat20:DEFERRED mixed:ADPT" local bytes
