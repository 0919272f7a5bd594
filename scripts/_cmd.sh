OUT=gpurun_out/r01_v19b; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
for tool in initcheck synccheck; do
  timeout 900 /usr/local/cuda/bin/compute-sanitizer --tool $tool --num-cuda-barriers 64 --error-exitcode 9 python scripts/sanitize_small.py > $OUT/sanitizer_$tool.log 2>&1
  echo "rc=$?" >> $OUT/sanitizer_$tool.log
done
