cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 300 python bench.py --workload c1 --steps 10 --warmup 3 --no-cpu --no-e2e > gpurun_out/bench_c1.json 2>>gpurun_out/bench.err
timeout 300 python bench.py --workload table2 --steps 10 --warmup 3 --no-cpu --no-e2e > gpurun_out/bench_table2.json 2>>gpurun_out/bench.err
timeout 300 python bench.py --workload c1 --steps 10 --warmup 3 --no-cpu --no-e2e --stage-events all > gpurun_out/bench_c1_all.json 2>>gpurun_out/bench.err
