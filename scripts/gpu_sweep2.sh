#!/bin/bash
# usage: scripts/gpu_sweep2.sh TAG "wl:versions ..."   e.g. "fem:25,30 stencil27_200:20"
cd $GRAFT_REPO_ROOT
TAG=$1; shift
OUT=gpurun_out/${TAG}
mkdir -p $OUT
timeout 900 python -m pytest tests -m gpu -x -q -k "not full_size" > $OUT/tests_small.log 2>&1
echo "rc=$?" >> $OUT/tests_small.log
for spec in $@; do
  wl=${spec%%:*}; vers=${spec#*:}
  for v in ${vers//,/ }; do
    TILESPMV_KERNEL=$v timeout 600 python bench.py --workload $wl --steps 200 --no-cpu-baseline --no-secondary --e2e-steps 2 \
       > $OUT/bench_v${v}_${wl}.json 2> $OUT/bench_v${v}_${wl}.err
  done
done
OUTG="$OUT/bench_v*.json" python - <<'PY' > $OUT/summary.txt
import json, glob, os
for f in sorted(glob.glob(os.environ["OUTG"])):
    try:
        d = json.loads(open(f).read().strip().splitlines()[-1])
        print(f, round(d["value"],1), "GF/s", round(d["kernel_ms"]["mean"],4), "ms", "frac", round(d["roofline"]["frac"],3))
    except Exception as e:
        print(f, "ERR", e)
PY
