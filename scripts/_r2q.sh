cd $GRAFT_REPO_ROOT
OUT=gpurun_out/r2q; mkdir -p $OUT
timeout 1500 python scripts/paper_ablation.py > $OUT/ablation.jsonl 2> $OUT/ablation.err
timeout 600 python scripts/cg_bench.py > $OUT/cg.json 2> $OUT/cg.err
timeout 300 python scripts/single_launch_diag.py fem > $OUT/single_fem.txt 2>&1
