cd $GRAFT_REPO_ROOT
NCU=/usr/local/cuda/bin/ncu
timeout 1200 $NCU --nvtx --nvtx-include "timed/" --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu > gpurun_out/launches_bench.log 2>&1
