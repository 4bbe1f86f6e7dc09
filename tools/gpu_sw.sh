cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 600 python -m pytest tests -m gpu -q -x -k "square" -p no:cacheprovider > gpurun_out/pytest_sq.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_sq.log
for r in 1 2; do timeout 300 python bench.py --workload c1 --steps 10 --warmup 3 --no-cpu --no-e2e >> gpurun_out/c1.txt 2>>gpurun_out/bench.err; done
timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu --no-e2e > gpurun_out/bench.json 2>>gpurun_out/bench.err
