cd $GRAFT_REPO_ROOT
OUT=gpurun_out/r2v; mkdir -p $OUT
timeout 600 python scripts/trace_items.py rmat20 > $OUT/trace_rmat20.txt 2>&1
timeout 600 python scripts/trace_items.py stencil27_200 > $OUT/trace_c5.txt 2>&1
timeout 600 python scripts/trace_items.py fem > $OUT/trace_fem.txt 2>&1
