cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
export SHAPES="[(128,9998),(9998,192),(256,14803),(14803,256),(192,9998),(9998,128),(14803,128),(64,9998)]"
export VARIANTS='[{"IPT_TILE_GROUP_TMA":0},{"IPT_DEBUG":1}]'
timeout 600 python tools/tile_big.py > gpurun_out/tile_diag.txt 2>&1
cat gpurun_out/tile_diag.txt
timeout 900 python -m pytest tests -m gpu -q -x --timeout 300 -p no:cacheprovider -k "group or tile or transpose" 2>&1 | tail -3
