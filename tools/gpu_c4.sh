cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
for r in 1 2; do timeout 600 python bench.py --workload c4 --steps 10 --warmup 3 --no-cpu --no-e2e > gpurun_out/bench_c4_$r.json 2>>gpurun_out/bench.err; done
IPT_CYC_SEG=2 timeout 600 python bench.py --workload c4 --steps 10 --warmup 3 --no-cpu --no-e2e --autotune 1 > gpurun_out/bench_c4_seg_model.json 2>>gpurun_out/bench.err
IPT_DEBUG=1 timeout 600 python bench.py --workload c4 --steps 2 --warmup 3 --no-cpu --no-e2e 2>&1 | grep -E "cycle_seg|autotune" | sort | uniq | head -30 > gpurun_out/c4_dbg.txt
