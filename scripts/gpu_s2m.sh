#!/bin/bash
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/s2m
for a in "l1.1x1a" "l4.1x1b" "l2.1x1a"; do
  timeout 300 ncu --set full --clock-control none --import-source on -k regex:k_tc_conv -s 2 -c 1 \
    -o gpurun_out/s2m/$a python scripts/one_layer.py $a 1 3 > gpurun_out/s2m/$a.log 2>&1
  ncu -i gpurun_out/s2m/$a.ncu-rep --page source --csv --print-source sass > gpurun_out/s2m/$a.src.csv 2>/dev/null
done
