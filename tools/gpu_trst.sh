cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/pytest_gpu.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_gpu.log
IPT_TILE_RESET=0 timeout 900 python -m pytest tests -m gpu -q -x -k "group or tile or 010" -p no:cacheprovider > gpurun_out/pytest_noreset.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_noreset.log
for r in 1 0 1 0; do IPT_TILE_RESET=$r timeout 300 python bench.py --workload table2 --steps 10 --warmup 3 --no-cpu --no-e2e >> gpurun_out/t2_rst.txt 2>>gpurun_out/bench.err; done
timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu --no-e2e > gpurun_out/bench.json 2>>gpurun_out/bench.err
