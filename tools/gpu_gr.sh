cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
for w in c1 table2 sweep; do for g in 0 1 0 1; do timeout 600 python bench.py --workload $w --steps 10 --warmup 3 --no-cpu --no-e2e --graphs $g >> gpurun_out/gr_$w.txt 2>>gpurun_out/bench.err; done; done
