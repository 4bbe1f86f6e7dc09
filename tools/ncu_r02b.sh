#!/bin/bash
# Second ncu batch for profiles/r02_*: the round-2 kernels in the bench's configurations.
set -x
NCU="ncu --set full --metrics lts__t_requests_op_atom.sum,lts__t_sectors_op_atom.sum,lts__t_requests_op_red.sum --clock-control none --import-source on -c 1"
P="python tools/prof_shape.py"
mkdir -p gpurun_out
# whole-GPU tiles: one C1 matrix (column split), Table 2 5100x2500 (row split)
$NCU -k regex:tile_group_rf -s 1 -o gpurun_out/r02_rf_c1 -f $P 1800 7200 --reps 1 > gpurun_out/ncu_rf_c1.log 2>&1
# unaligned segmented walker: 9797x13081 stage 1 (412-byte units, the bench's tuned plan) and 5735x6925 (5540 B)
$NCU -k regex:cycle_seg_ua -s 0 -o gpurun_out/r02_seg_ua -f $P 9797 13081 --m 9797 --n 103 --reps 1 > gpurun_out/ncu_segua.log 2>&1
$NCU -k regex:cycle_seg_ua -s 0 -o gpurun_out/r02_seg_ua_big -f $P 5735 6925 --m 5735 --n 1385 --reps 1 > gpurun_out/ncu_segua2.log 2>&1
# element-path group tiles, column split (the slow random-shape class): 4096x9998 with 256x9998 tiles
$NCU -k regex:tile_group_generic -s 0 -o gpurun_out/r02_tile_generic_cs -f $P 4096 9998 --m 256 --n 9998 --reps 1 > gpurun_out/ncu_tgcs.log 2>&1
# launch list of the default bench headline (C5), shares of the step
ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/launches_c5.csv python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu --sub none > gpurun_out/ncu_launch_c5.log 2>&1
