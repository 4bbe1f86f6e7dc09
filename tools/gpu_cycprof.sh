cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/ncu
timeout 600 ncu --set full --import-source on --clock-control none -k regex:cycle_global --launch-skip 2 -c 1 -o gpurun_out/ncu/cyc_S256 -f python tools/cyc_one.py 1 16384 256 64 2 > /dev/null 2>&1
timeout 600 ncu --set full --import-source on --clock-control none -k regex:cycle_global --launch-skip 2 -c 1 -o gpurun_out/ncu/cyc_S1024 -f python tools/cyc_one.py 1 16384 64 256 2 > /dev/null 2>&1
ls gpurun_out/ncu
