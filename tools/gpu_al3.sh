cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
export SHAPES="[(192,9998),(128,9998),(64,9998),(64,14803),(128,14803),(256,14803)]"
export VARIANTS='[{},{"IPT_TILE_GROUP_TMA_GENERIC":1,"IPT_DEBUG":1},{},{"IPT_TILE_GROUP_TMA_GENERIC":1}]'
timeout 900 python tools/tile_big.py > gpurun_out/tile_big.txt 2>&1
