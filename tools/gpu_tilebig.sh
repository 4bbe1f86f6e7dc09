cd $GRAFT_REPO_ROOT
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x --timeout 300 -p no:cacheprovider -k "010" > gpurun_out/pytest_gpu.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_gpu.log
export SHAPES="[(8192,113),(9998,64),(14803,32),(64,9998),(4999,32),(8192,131)]"
timeout 300 python tools/tile_sweep.py > gpurun_out/tile_sweep.log 2>&1
