cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/pytest_gpu.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_gpu.log
IPT_TILE_GEN_TMAA=0 timeout 600 python -m pytest tests -m gpu -q -x -k "element or group" -p no:cacheprovider > gpurun_out/pytest_notmaa.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_notmaa.log
timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu --no-e2e > gpurun_out/bench.json 2>>gpurun_out/bench.err
