OUT=gpurun_out/r01_v18; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 900 python -m pytest tests -m gpu -x -q > $OUT/tests_gpu.log 2>&1; echo "rc=$?" >> $OUT/tests_gpu.log
python scripts/ab_bench.py rmat20 40,42,40@LOCAL_PARTS=8 --rounds 3 --steps 50 > $OUT/ab_rmat.txt 2>&1
python scripts/ab_bench.py mixed 40,42 --rounds 3 --steps 50 > $OUT/ab_mixed.txt 2>&1
python scripts/trace_items.py rmat20 > $OUT/trace_rmat20.txt 2>&1
