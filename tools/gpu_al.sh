cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 600 python -m pytest tests -m gpu -q -x -k "element or group or 010 or sweep_f32 or autotuned" -p no:cacheprovider > gpurun_out/pytest_al.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_al.log
export SHAPES="[(9998,192),(9998,128),(14803,128),(14803,256),(4999,96),(192,9998),(64,14803)]"
export VARIANTS='[{"IPT_TILE_GEN_TMAA":0},{"IPT_TILE_GEN_TMAA":1,"IPT_DEBUG":1},{"IPT_TILE_GEN_TMAA":0},{"IPT_TILE_GEN_TMAA":1}]'
timeout 900 python tools/tile_big.py > gpurun_out/tile_big.txt 2>&1
