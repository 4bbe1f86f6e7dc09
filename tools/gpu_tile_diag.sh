cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
export SHAPES="[(256,15000),(240,7200),(7200,240),(64,16384),(15000,256),(384,10000),(20000,200),(192,9998),(10000,384),(14803,256),(256,14803),(9998,192)]"
export VARIANTS='[{},{"IPT_TILE_GROUP_PERSM":2,"IPT_DEBUG":1}]'
timeout 600 python tools/tile_big.py > gpurun_out/tile_diag.txt 2>&1
cat gpurun_out/tile_diag.txt
