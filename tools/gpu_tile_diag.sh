cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
export SHAPES="[(256,15000),(240,7200),(7200,240),(64,16384),(384,10000),(20000,200),(10000,384),(15000,256),(128,16384),(100,20000),(200,20000),(160,20000)]"
export VARIANTS='[{"IPT_TILE_GROUP_TMA":0},{"IPT_DEBUG":1}]'
timeout 600 python tools/tile_big.py > gpurun_out/tile_diag.txt 2>&1
cat gpurun_out/tile_diag.txt
timeout 900 python -m pytest tests -m gpu -q -x --timeout 300 -p no:cacheprovider -k "tile or group or transpose or plan" 2>&1 | tail -3
