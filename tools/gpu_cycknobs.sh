cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
export CASES="[('pow2_S256', (1, 256, 16384, 64)), ('S800', (1, 10000, 100, 200)), ('S960', (1, 7200, 75, 240)), ('S1024', (1, 15000, 50, 256)), ('S768', (1, 9998, 64, 192))]"
export KNOBS="[{}, {'IPT_CYC_G':'8','IPT_CYC_R':'2'}, {'IPT_CYC_G':'4','IPT_CYC_R':'4'}, {'IPT_CYC_G':'16','IPT_CYC_R':'2'}, {'IPT_CYC_G':'8','IPT_CYC_R':'4'}, {'IPT_CYC_MAXVEC':'32'}, {'IPT_CYC_BLOCKS_PER_SM':'6'}, {'IPT_CYC_FENCE':'0'}]"
timeout 600 python tools/cyc_knobs.py 2>&1 | tail -12
