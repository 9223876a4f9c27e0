#!/bin/bash
# fix check: the pair's out-of-range M tile no longer stores (GEMM aliasing onto rows 0..127)
nvidia-smi --query-gpu=uuid --format=csv,noheader > gpurun_out/fix1_box.txt
for i in 1 2 3; do
  for v in ALT_TC_ROUND=0 ALT_TC_ROUND=1; do
    env $v python -m pytest tests/test_gpu_conv3d.py tests/test_gpu_conv.py tests/test_gpu_store_at.py -q --timeout 900 -p no:cacheprovider > gpurun_out/fix1_${v}_$i.txt 2>&1
  done
done
python -m pytest tests -m gpu -q --timeout 1500 -p no:cacheprovider > gpurun_out/fix1_full.txt 2>&1
