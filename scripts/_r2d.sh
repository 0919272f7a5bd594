cd $GRAFT_REPO_ROOT
bash scripts/gpu_ab.sh r2d "rmat20:DEFERRED mixed:DEFERRED mixed:ADPT stencil27_200:DEFERRED" d2i d2i_med d3 r01_head
