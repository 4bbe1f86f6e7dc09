# Full GPU session: tests, smoke, bench (all workloads), ncu launch lists + full captures.
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
NCU=/usr/local/cuda/bin/ncu
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
timeout 1500 python -m pytest tests -m gpu -q --timeout 300 -p no:cacheprovider > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 900 python bench.py --steps 10 --warmup 3 > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?" >> gpurun_out/bench.err
for w in c1 c3 c4 c5 table2; do timeout 600 python bench.py --workload $w --steps 10 --warmup 3 --no-cpu > gpurun_out/bench_$w.json 2>> gpurun_out/bench.err; done
timeout 600 python bench.py --impl reference --steps 2 --warmup 3 > gpurun_out/bench_ref.json 2>> gpurun_out/bench.err
# launch lists (cold, serialised) of the bench commands: every kernel with its time and DRAM bytes
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum
timeout 1200 $NCU --nvtx --nvtx-include "timed/" --metrics $M --clock-control none --csv --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu > gpurun_out/launches_bench.log 2>&1
for w in c1 c3 c4 c5; do
  timeout 900 $NCU --nvtx --nvtx-include "timed/" --metrics $M --clock-control none --csv --log-file gpurun_out/launches_$w.csv python bench.py --workload $w --steps 2 --warmup 3 --no-e2e --no-cpu > gpurun_out/launches_bench_$w.log 2>&1
done
# one full capture of each kernel kind on sweep matrices (12800x15000 and 9998x12288 plans)
IPT_CYC_SEG=0 timeout 900 $NCU --set full --clock-control none --import-source on -k regex:cycle_global -s 1 -c 1 -o gpurun_out/prof_cyc -f python tools/prof_one.py 12800 15000 2 > gpurun_out/prof_cyc.log 2>&1
timeout 600 $NCU --set full --clock-control none --import-source on -k regex:tile_ -s 2 -c 1 -o gpurun_out/prof_tile -f python tools/prof_one.py 12800 15000 2 > gpurun_out/prof_tile.log 2>&1
timeout 600 $NCU --set full --clock-control none --import-source on -k regex:tile_ -s 2 -c 1 -o gpurun_out/prof_tile_generic -f python tools/prof_one.py 9998 12288 2 > gpurun_out/prof_tile_generic.log 2>&1
timeout 600 $NCU --set full --clock-control none --import-source on -k regex:square_swap -s 1 -c 1 -o gpurun_out/prof_sq -f python tools/prof_one.py 16384 16384 2 > gpurun_out/prof_sq.log 2>&1
timeout 900 $NCU --set full --clock-control none --import-source on -k regex:cycle_seg -s 1 -c 1 -o gpurun_out/prof_seg -f python tools/prof_one.py 20000 30000 2 8 > gpurun_out/prof_seg.log 2>&1
ls gpurun_out
