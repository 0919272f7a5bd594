#!/bin/bash
# usage: scripts/gpu_sweep.sh TAG "kernel versions" "workloads"
cd $GRAFT_REPO_ROOT
TAG=$1; VERS=${2:-"2"}; WLS=${3:-"stencil27_200 fem"}
OUT=gpurun_out/${TAG}
mkdir -p $OUT
timeout 900 python -m pytest tests -m gpu -x -q -k "not full_size" > $OUT/tests_small.log 2>&1
echo "rc=$?" >> $OUT/tests_small.log
for v in $VERS; do
  for wl in $WLS; do
    TILESPMV_KERNEL=$v timeout 600 python bench.py --workload $wl --steps 200 --no-cpu-baseline --no-secondary --e2e-steps 2 \
       > $OUT/bench_v${v}_${wl}.json 2> $OUT/bench_v${v}_${wl}.err
  done
done
python - <<'PY' > $OUT/summary.txt
import json, glob, os
for f in sorted(glob.glob(os.environ.get("OUTG","") or "gpurun_out/*/bench_v*.json")):
    try:
        d = json.loads(open(f).read().strip().splitlines()[-1])
        print(f, round(d["value"],1), "GF/s", round(d["kernel_ms"]["mean"],4), "ms", "frac", round(d["roofline"]["frac"],3))
    except Exception as e:
        print(f, "ERR", e)
PY
