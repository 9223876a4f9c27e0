#!/bin/bash
# knob bisection of the first-launch residual loss (flow: test_gpu_store_at.py alone)
for v in ALT_X=0 ALT_TC_RES_MODE=4 ALT_TC_KNOB=1 ALT_TC_KNOB=2 ALT_PDL=0; do
  for i in 1 2 3; do
    env $v python -m pytest tests/test_gpu_store_at.py -q --timeout 900 -p no:cacheprovider > gpurun_out/fl4_${v}_$i.txt 2>&1
  done
done
