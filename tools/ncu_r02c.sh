#!/bin/bash
# Third ncu batch for profiles/r02_* (late round 2): the rf kernel in both C5 orientations
# (row split 4096x3000, column split 3000x4096), the element-path group kernel on a 2-D
# slice grid (1279x6353 tiles of 15348x19059), and the headline launch list.
set -x
NCU="ncu --set full --clock-control none --import-source on"
P="python tools/prof_shape.py"
mkdir -p gpurun_out
$NCU -k regex:tile_group_rf -s 2 -c 2 -o gpurun_out/r02_rf_ab -f $P 4096 3000 --count 64 --m 4096 --n 3000 --reps 2 > gpurun_out/ncu_rf_ab.log 2>&1
$NCU -k regex:tile_group_generic -s 0 -c 1 -o gpurun_out/r02_tile_generic_2d -f $P 15348 19059 --m 1279 --n 6353 --reps 1 > gpurun_out/ncu_tg2d.log 2>&1
ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/launches_c5.csv python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu --sub none --autotune 1 > gpurun_out/ncu_launch_c5.log 2>&1
