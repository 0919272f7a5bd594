cd $GRAFT_REPO_ROOT
bash scripts/gpu_ab.sh r2x "rmat20:DEFERRED" gc0 gc160 gc320 gc640
