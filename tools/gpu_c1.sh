cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 600 python -m pytest tests -m gpu -q -x -k "autotune or C1 or cycle_seg or graph" -p no:cacheprovider > gpurun_out/pytest_gpu.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_gpu.log
timeout 300 python bench.py --workload c1 --steps 10 --warmup 3 --no-cpu --no-e2e > gpurun_out/bench_c1.json 2>gpurun_out/bench.err
