cd $GRAFT_REPO_ROOT
bash scripts/gpu_ab.sh r2y "rmat20:DEFERRED mixed:DEFERRED stencil27_200:DEFERRED" gc320 gc320_1024 gc320_4096 gc480_2048 gc320_3072
