cd $GRAFT_REPO_ROOT
timeout 600 python tools/tile_sweep.py > gpurun_out/tile_sweep.log 2>&1
timeout 600 python bench.py --steps 10 --warmup 3 --e2e-steps 2 > gpurun_out/bench.json 2> gpurun_out/bench.err
echo "bench rc=$?" >> gpurun_out/bench.err
