cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
export SHAPES="[(9998,192),(9998,128),(14803,128),(14803,256),(256,15000),(64,15000),(7200,240)]"
export VARIANTS='[{},{"IPT_TILE_GROUP_NBUF":3},{},{"IPT_TILE_GROUP_NBUF":3}]'
timeout 900 python tools/tile_big.py > gpurun_out/tile_big.txt 2>&1
