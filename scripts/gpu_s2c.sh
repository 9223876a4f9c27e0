#!/bin/bash
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/s2c
for a in "l4.3x3 1" "l4.3x3 4" "l1.3x3 1"; do
  set -- $a
  timeout 300 ncu --set full --clock-control none --import-source on -k regex:k_tc_conv -s 2 -c 1 \
    -o gpurun_out/s2c/$1_s$2 python scripts/one_layer.py $1 $2 3 > gpurun_out/s2c/$1_s$2.log 2>&1
  python scripts/one_layer.py $1 $2 3 2>&1 | tail -1
done
