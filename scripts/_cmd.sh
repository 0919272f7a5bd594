OUT=gpurun_out/r01_v16; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 900 python -m pytest tests -m gpu -x -q > $OUT/tests_gpu.log 2>&1; echo "rc=$?" >> $OUT/tests_gpu.log
python scripts/ab_bench.py stencil27_200 20,40,42 --rounds 3 --steps 20 > $OUT/ab_stencil.txt 2>&1
python scripts/ab_bench.py rmat20 20,40,42 --rounds 3 --steps 50 > $OUT/ab_rmat.txt 2>&1
python scripts/ab_bench.py mixed 20,40,42 --rounds 3 --steps 50 > $OUT/ab_mixed.txt 2>&1
python scripts/ab_bench.py mixed 20,40,42 --mode ADPT --rounds 3 --steps 50 > $OUT/ab_mixed_adpt.txt 2>&1
python scripts/ab_bench.py fem 25,41,40 --rounds 3 --steps 100 > $OUT/ab_fem.txt 2>&1
