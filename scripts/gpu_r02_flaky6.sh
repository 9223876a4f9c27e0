#!/bin/bash
for m in FLAKE_SYNC=1 FLAKE_X=0; do
  for i in 1 2 3 4 5 6; do
    env $m python -m pytest tests/test_gpu_store_at.py -q --timeout 900 -p no:cacheprovider > gpurun_out/fl6_${m}_$i.txt 2>&1
  done
done
