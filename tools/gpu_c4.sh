cd $GRAFT_REPO_ROOT
for i in 1 2 3; do timeout 600 python bench.py --workload c4 --steps 10 --warmup 3 --no-cpu --no-e2e > gpurun_out/bench_c4_$i.json 2>/dev/null; done
