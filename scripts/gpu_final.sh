#!/bin/bash
# Round-end evidence: scripts/gpu_round.sh TAG, then the paper ablation and the CG bench.
cd $GRAFT_REPO_ROOT
TAG=${1:-final}
bash scripts/gpu_round.sh $TAG
OUT=gpurun_out/$TAG
timeout 1500 python scripts/paper_ablation.py > $OUT/ablation.jsonl 2> $OUT/ablation.err
timeout 300 python scripts/cg_bench.py > $OUT/cg.jsonl 2> $OUT/cg.err
echo done > $OUT/DONE2
