#!/bin/bash
# intermittent store_at TC failure: residual-load variants (ALT_TC_RES_MODE) and PDL off
for v in "ALT_TC_RES_MODE=0" "ALT_TC_RES_MODE=1" "ALT_TC_RES_MODE=2" "ALT_PDL=0"; do
  for i in 1 2 3 4; do
    env $v python -m pytest tests/test_gpu_fullsize.py tests/test_gpu_store_at.py -q --timeout 900 -p no:cacheprovider \
      -k "b1_tuned or parity" > gpurun_out/fl_${v}_$i.txt 2>&1
  done
done
