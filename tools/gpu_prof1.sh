cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
NCU=/usr/local/cuda/bin/ncu
timeout 600 $NCU --set full --clock-control none --import-source on -k regex:tile_onchip -s 1 -c 1 -o gpurun_out/prof_tile -f python tools/prof_one.py 12800 15000 1 > gpurun_out/prof_tile.log 2>&1
timeout 900 $NCU --set full --clock-control none --import-source on -k regex:cycle_global -s 2 -c 2 -o gpurun_out/prof_cyc -f python tools/prof_one.py 12800 15000 1 > gpurun_out/prof_cyc.log 2>&1
timeout 900 $NCU --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu > gpurun_out/launches_bench.log 2>&1
ls -la gpurun_out
