cd $GRAFT_REPO_ROOT
nvidia-smi -L > gpurun_out/g1_smi.txt 2>&1
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/g1_smoke.log 2>&1
echo "smoke rc=$?" >> gpurun_out/g1_smoke.log
timeout 900 python -m pytest tests -m gpu -x -q -k "not full_size" > gpurun_out/g1_tests_small.log 2>&1
echo "rc=$?" >> gpurun_out/g1_tests_small.log
timeout 600 python bench.py --steps 100 --no-secondary --cpu-seconds 3 > gpurun_out/g1_bench.json 2> gpurun_out/g1_bench.err
echo "rc=$?" >> gpurun_out/g1_bench.err
timeout 1200 python -m pytest tests -m gpu -x -q -k "full_size" > gpurun_out/g1_tests_full.log 2>&1
echo "rc=$?" >> gpurun_out/g1_tests_full.log
