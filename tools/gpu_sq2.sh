cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
export SHAPES='[(16384,4),(20000,4),(1024,4),(512,4),(20000,8),(8192,8),(1024,8)]'
export VARIANTS='[{"IPT_DEBUG":1},{"IPT_SQ_TB":256},{"IPT_SQ_TB":512}]'
timeout 600 python tools/sq_sweep.py > gpurun_out/sq_sweep.txt 2>&1
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/pytest_gpu.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_gpu.log
timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu --no-e2e > gpurun_out/bench.json 2>gpurun_out/bench.err
