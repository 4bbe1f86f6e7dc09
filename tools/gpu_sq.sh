cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
export SHAPES="${SHAPES:-[(16384,4),(20000,4),(10007,4),(8192,4),(4096,4),(1024,4),(256,4),(20000,8),(8192,8)]}"
[ -n "$VARIANTS" ] || export VARIANTS='[{"IPT_DEBUG":1},{"IPT_SQ_TB":512},{"IPT_SQ_ELEM":1}]'

timeout 900 python tools/sq_sweep.py > gpurun_out/sq_sweep.txt 2>&1
timeout 600 python -m pytest tests -m gpu -q -x -k "square or small_shapes or 010 or sweep_f32" -p no:cacheprovider > gpurun_out/pytest_sq.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_sq.log
timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu --no-e2e > gpurun_out/bench.json 2>gpurun_out/bench.err
