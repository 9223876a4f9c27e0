#!/bin/bash
# first-GEMM residual loss vs CUDA module loading mode
for m in LAZY EAGER; do
  for i in 1 2 3 4 5 6; do
    CUDA_MODULE_LOADING=$m python -m pytest tests/test_gpu_store_at.py -q --timeout 900 -p no:cacheprovider > gpurun_out/fl5_${m}_$i.txt 2>&1
  done
done
