cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
export SHAPES='[(1024,4),(1800,4),(2048,4),(3072,4),(4096,4),(8192,4)]'
export VARIANTS='[{"IPT_SQ_SWZ":0},{"IPT_SQ_SWZ":1},{"IPT_SQ_SWZ":0,"IPT_SQ_TB":256},{"IPT_SQ_SWZ":1,"IPT_SQ_TB":256},{"IPT_SQ_SWZ":0},{"IPT_SQ_SWZ":1}]'
timeout 900 python tools/sq_sweep.py > gpurun_out/sq_sweep.txt 2>&1
