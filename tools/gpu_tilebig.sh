cd $GRAFT_REPO_ROOT
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x --timeout 300 -p no:cacheprovider -k "010" > gpurun_out/pytest_gpu.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_gpu.log
export SHAPES="[(120,7200),(64,10000),(7200,120),(256,200),(400,400),(160,1800)]"
IPT_TILE_STREAM=0 timeout 300 python tools/tile_sweep.py > gpurun_out/tile_sweep.log 2>&1
IPT_TILE_STREAM=1 timeout 300 python tools/tile_sweep.py >> gpurun_out/tile_sweep.log 2>&1
