#!/bin/bash
# ncu captures for profiles/r02_* (run under gpurun from the repo root).  One kernel per
# capture (-k regex, -s skips the autotune / warm-up launches), --set full plus the L2
# atomic counters; summarised by tools/summarize_ncu.py.
set -x
NCU="ncu --set full --metrics lts__t_requests_op_atom.sum,lts__t_sectors_op_atom.sum,lts__t_requests_op_red.sum,lts__t_sectors_op_red.sum,l1tex__t_requests_pipe_lsu_mem_global_op_atom.sum --clock-control none --import-source on -c 1"
P="python tools/prof_shape.py"
mkdir -p gpurun_out
# headline C5 (512 x 4096 x 3000 f32, the bench's tuned batch plans): stage kernels
$NCU -k regex:cycle_seg -s 0 -o gpurun_out/r02_c5_cycle_seg -f $P 4096 3000 --count 512 --reps 1 --m 256 --n 3000 > gpurun_out/ncu_c5a.log 2>&1
$NCU -k regex:tile_group -s 0 -o gpurun_out/r02_c5_tile -f $P 4096 3000 --count 512 --reps 1 --m 256 --n 3000 > gpurun_out/ncu_c5b.log 2>&1
# flag-based PTTWAC on a sweep stage (18000 x 7200: 384-byte units) -- claim atomics
IPT_CYC_SEG=0 $NCU -k regex:cycle_global -s 0 -o gpurun_out/r02_cycle_global -f $P 18000 7200 --m 18000 --n 96 --reps 1 > gpurun_out/ncu_cg.log 2>&1
# realigning walker (9797 x 13081: 508-byte units)
$NCU -k regex:cycle_ua -s 0 -o gpurun_out/r02_cycle_ua -f $P 9797 13081 --m 9797 --n 127 --reps 1 > gpurun_out/ncu_ua.log 2>&1
# element-path group tile (same shape)
$NCU -k regex:tile_group_generic -s 0 -o gpurun_out/r02_tile_generic -f $P 9797 13081 --m 9797 --n 127 --reps 1 > gpurun_out/ncu_tg.log 2>&1
# segmented cycles on C4 (20000 x 30000 f64, 256-byte units)
$NCU -k regex:cycle_seg -s 0 -o gpurun_out/r02_c4_cycle_seg -f $P 20000 30000 --eb 8 --m 32 --n 30000 --reps 1 > gpurun_out/ncu_c4.log 2>&1
# element-path square swap (10007^2 f32)
$NCU -k regex:square_swap -s 0 -o gpurun_out/r02_square_elem -f $P 10007 10007 --reps 1 > gpurun_out/ncu_sq.log 2>&1
# scalar fallback (10007 x 19997 f32, 4-byte units, per-lane walkers)
$NCU -k regex:cycle_global -s 0 -o gpurun_out/r02_scalar -f $P 10007 19997 --reps 1 > gpurun_out/ncu_scalar.log 2>&1
# launch list of the default bench headline (timed share check)
ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/launches_c5.csv python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu --sub none > gpurun_out/ncu_launch_c5.log 2>&1
