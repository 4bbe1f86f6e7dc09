cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 300 python bench.py --workload c1 --steps 10 --warmup 3 --no-cpu --no-e2e > gpurun_out/bench_c1.json 2>gpurun_out/bench.err
timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu --no-e2e > gpurun_out/bench.json 2>>gpurun_out/bench.err
for w in c3 c4 c5; do timeout 600 python bench.py --workload $w --steps 10 --warmup 3 --no-cpu --no-e2e > gpurun_out/bench_$w.json 2>>gpurun_out/bench.err; done
