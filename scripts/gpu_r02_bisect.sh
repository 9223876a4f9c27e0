#!/bin/bash
# per-kernel ncu durations of one R50 step for each round-2 commit touching tc_conv.cu (regression bisection)
nvidia-smi --query-gpu=uuid --format=csv,noheader > gpurun_out/bis_box.txt
R=$(pwd)
for d in .r01 .bis_1b6b138 .bis_b396dfa .bis_41191af .bis_17ca455 .bis_0a32ec1 .; do
  n=$(basename $d); [ "$d" = . ] && n=cur
  (cd $d && ncu --metrics gpu__time_duration.sum --clock-control none -k regex:k_tc_conv --csv --log-file $R/gpurun_out/bis_$n.csv python scripts/one_step_r50.py > $R/gpurun_out/bis_$n.log 2>&1)
done
