cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 600 python bench.py --workload table2 --steps 10 --warmup 3 --no-cpu > gpurun_out/bench_table2.json 2>>gpurun_out/bench.err
timeout 600 python bench.py --workload table2 --steps 10 --warmup 3 --no-cpu --no-e2e --algo 4stage > gpurun_out/bench_table2_4stage.json 2>>gpurun_out/bench.err
timeout 900 python bench.py --steps 6 --warmup 3 --no-cpu --no-e2e --algo 4stage > gpurun_out/bench_4stage.json 2>>gpurun_out/bench.err
