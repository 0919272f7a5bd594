#!/bin/bash
# GPU tests on the in-tree build, then an in-process A/B of library builds
# (scripts/ab_libs.py).  usage: scripts/gpu_ablibs.sh TAG "wl:mode,..." "ab_old/a.so,ab_old/b.so" [pytest args]
cd $GRAFT_REPO_ROOT
TAG=$1; WLS=$2; LIBS=$3; shift 3
OUT=gpurun_out/$TAG; mkdir -p $OUT
if [ "$1" != "notest" ]; then
  timeout 900 python -m pytest tests -m gpu -x -q "$@" > $OUT/tests_gpu.log 2>&1; echo "rc=$?" >> $OUT/tests_gpu.log
fi
timeout 1500 python scripts/ab_libs.py "$WLS" "$LIBS" > $OUT/ab.txt 2> $OUT/ab.err; echo "rc=$?" >> $OUT/ab.txt
