cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
for a in 4 8 16; do timeout 900 python bench.py --steps 10 --warmup 3 --no-cpu --no-e2e --autotune $a > gpurun_out/bench_at$a.json 2>>gpurun_out/bench.err; done
for a in 4 12; do timeout 900 python bench.py --workload c3 --steps 10 --warmup 3 --no-cpu --no-e2e --autotune $a > gpurun_out/bench_c3_at$a.json 2>>gpurun_out/bench.err; done
