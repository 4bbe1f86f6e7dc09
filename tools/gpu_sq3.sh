cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 300 python -m pytest tests -m gpu -q -x -k "square" -p no:cacheprovider > gpurun_out/pytest_sq.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_sq.log
export SHAPES='[(16384,4),(20000,4),(8192,4),(1024,4),(20000,8),(8192,8),(1024,16)]'
export VARIANTS='[{"IPT_SQ_SWZ":0},{"IPT_SQ_SWZ":1},{"IPT_SQ_SWZ":0},{"IPT_SQ_SWZ":1}]'
timeout 900 python tools/sq_sweep.py > gpurun_out/sq_sweep.txt 2>&1
