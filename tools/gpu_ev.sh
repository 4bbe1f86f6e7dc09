cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
for m in all last none all last none; do timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu --no-e2e --stage-events $m > gpurun_out/bench_ev_$m.json 2>>gpurun_out/bench.err; cat gpurun_out/bench_ev_$m.json >> gpurun_out/ev_all.txt; done
for m in all last; do timeout 600 python bench.py --workload table2 --steps 10 --warmup 3 --no-cpu --no-e2e --stage-events $m >> gpurun_out/ev_t2.txt 2>>gpurun_out/bench.err; done
