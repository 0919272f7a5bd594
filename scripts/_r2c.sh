cd $GRAFT_REPO_ROOT
OUT=gpurun_out/r2c; mkdir -p $OUT
PKG=paper_conf_ipps_niuldj0t21_b200
for wl in lap2d_64 fem; do timeout 300 python scripts/single_launch_diag.py $wl > $OUT/single_$wl.txt 2>&1; done
NCU=/usr/local/cuda/bin/ncu
for v in d3 r01_head; do
  cp ab_old/$v.so $PKG/libtilespmv.so; touch $PKG/libtilespmv.so
  for wl in rmat20 mixed; do
    timeout 900 $NCU --set full --clock-control none --import-source on -k regex:tilespmv_fp64 -s 3 -c 1 \
      -o $OUT/full_${v}_${wl} -f python bench.py --workload $wl --steps 2 --warmup 3 --no-cpu-baseline \
      --no-secondary --e2e-steps 0 > $OUT/full_${v}_${wl}.log 2>&1
  done
done
cp ab_old/d3.so $PKG/libtilespmv.so; touch $PKG/libtilespmv.so
