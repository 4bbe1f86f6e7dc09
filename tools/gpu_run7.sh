cd $GRAFT_REPO_ROOT
timeout 1500 python -m pytest tests -m gpu -q --timeout 300 -p no:cacheprovider > gpurun_out/pytest_gpu.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_gpu.log
timeout 600 python bench.py --steps 6 --warmup 3 --no-e2e --no-cpu --algo 4stage > gpurun_out/bench_4stage.json 2> gpurun_out/bench.err
timeout 600 python bench.py --steps 6 --warmup 3 --no-e2e --no-cpu > gpurun_out/bench.json 2>> gpurun_out/bench.err
