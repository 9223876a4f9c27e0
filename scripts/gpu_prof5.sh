#!/bin/bash
make -C paper_conf_eurosys_xuxpwwwdxcwc23_b200 -j8 >/dev/null 2>&1
mkdir -p gpurun_out/prof5
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_tc_conv -s 1 -c 1 \
  -o gpurun_out/prof5/epi python scripts/exp_epi1.py > gpurun_out/prof5/ncu.log 2>&1
ncu -i gpurun_out/prof5/epi.ncu-rep --page source --csv --print-source sass > gpurun_out/prof5/sass.csv 2>&1
