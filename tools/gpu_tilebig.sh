cd $GRAFT_REPO_ROOT
export SHAPES="[(7200,120),(10000,64),(120,7200),(256,200)]"
for g in 0 8 16 32 0; do IPT_TILE_GROUP=$g timeout 300 python tools/tile_sweep.py | sed "s/^/GB=$g /" >> gpurun_out/tile_sweep.log 2>&1; done
