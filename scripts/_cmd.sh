OUT=gpurun_out/r01_n2; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
for ex in halo allgather; do
TILESPMV_BENCH_ONE_GPU=1 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29511 bench.py --gpus 2 --steps 10 --warmup 3 --workload stencil27_200 --exchange $ex --e2e-steps 2 > $OUT/n2_$ex.json 2> $OUT/n2_$ex.err
echo "rc=$?" >> $OUT/n2_$ex.err
done
