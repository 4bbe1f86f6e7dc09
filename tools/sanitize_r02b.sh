set -x
CS="compute-sanitizer --print-limit 20"
IPT_TILE_RF_FORCE=1 timeout 900 $CS --tool memcheck python tools/prof_shape.py 600 4096 --m 600 --n 4096 --count 2 --reps 1 > gpurun_out/san1.log 2>&1; echo "rc=$?" >> gpurun_out/san1.log
IPT_TILE_RF_FORCE=1 timeout 900 $CS --tool racecheck python tools/prof_shape.py 600 4096 --m 600 --n 4096 --reps 1 > gpurun_out/san2.log 2>&1; echo "rc=$?" >> gpurun_out/san2.log
IPT_TILE_GROUP_COLSPLIT=2 timeout 900 $CS --tool memcheck python tools/prof_shape.py 1202 2406 --m 601 --n 1203 --reps 1 > gpurun_out/san3.log 2>&1; echo "rc=$?" >> gpurun_out/san3.log
IPT_TILE_GROUP_COLSPLIT=2 timeout 900 $CS --tool racecheck python tools/prof_shape.py 1202 2406 --m 601 --n 1203 --reps 1 > gpurun_out/san4.log 2>&1; echo "rc=$?" >> gpurun_out/san4.log
IPT_CYC_SEG=2 timeout 900 $CS --tool memcheck python tools/prof_shape.py 9797 13081 --m 9797 --n 127 --reps 1 > gpurun_out/san5.log 2>&1; echo "rc=$?" >> gpurun_out/san5.log
IPT_CYC_SEG=2 timeout 900 $CS --tool memcheck python tools/prof_shape.py 382 1530 --m 382 --n 765 --reps 1 > gpurun_out/san6.log 2>&1; echo "rc=$?" >> gpurun_out/san6.log
