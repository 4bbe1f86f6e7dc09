# Tile-stage experiments on the sweep's panel tiles + one source-level ncu capture.
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
export SHAPES="[(256,15000),(240,7200),(7200,240),(64,16384),(15000,256),(384,10000),(20000,200),(192,9998)]"
export VARIANTS='[{"IPT_DEBUG":1},{"IPT_TILE_GROUP_COLSPLIT":1},{"IPT_TILE_GROUP_COLSPLIT":0},{"IPT_TILE_GROUP_NBUF":3},{"IPT_TILE_SMEM_MAX":150000}]'
timeout 900 python tools/tile_big.py > gpurun_out/tile_exp.txt 2>&1
NCU=/usr/local/cuda/bin/ncu
timeout 600 $NCU --set full --clock-control none --import-source on -k regex:tile_ -s 2 -c 1 -o gpurun_out/prof_tile -f python tools/prof_one.py 12800 15000 2 > gpurun_out/prof_tile.log 2>&1
timeout 600 $NCU --set full --clock-control none --import-source on -k regex:tile_ -s 2 -c 1 -o gpurun_out/prof_tile_row -f python tools/prof_one.py 7200 18000 2 > gpurun_out/prof_tile_row.log 2>&1
ls gpurun_out
