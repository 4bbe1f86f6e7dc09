cd $GRAFT_REPO_ROOT
export SHAPES="${SHAPES:-[(120,7200),(7200,120),(60,12800),(12800,60),(64,10000),(10000,64),(32,20000),(20000,32),(256,256)]}"
export VARIANTS="${VARIANTS:-[{\"IPT_DEBUG\":1}]}"
timeout 900 python tools/tile_big.py > gpurun_out/tile_big.txt 2>&1
