cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 600 python -m pytest tests -m gpu -q -x -k "seg or graph or C1 or 100" -p no:cacheprovider > gpurun_out/pytest_rst.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_rst.log
for r in 1 0 1 0; do IPT_SEG_RESET=$r timeout 300 python bench.py --workload c1 --steps 10 --warmup 3 --no-cpu --no-e2e >> gpurun_out/c1_rst.txt 2>>gpurun_out/bench.err; done
