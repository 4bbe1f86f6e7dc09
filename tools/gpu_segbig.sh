cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
for w in c3 c4; do
  timeout 600 python bench.py --workload $w --steps 6 --warmup 3 --no-cpu --no-e2e > gpurun_out/bench_${w}_flags.json 2>>gpurun_out/bench.err
  IPT_CYC_SEG=2 IPT_CYC_SEG_MAX_MB=100000 timeout 600 python bench.py --workload $w --steps 6 --warmup 3 --no-cpu --no-e2e > gpurun_out/bench_${w}_seg.json 2>>gpurun_out/bench.err
done
