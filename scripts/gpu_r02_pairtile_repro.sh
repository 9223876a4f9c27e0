#!/bin/bash
# reproducer of the pair-tile aliasing race (test_matmul_store_at_parity[384x192x256p7tc-bf16]): fresh processes, both epilogue store modes
nvidia-smi --query-gpu=uuid --format=csv,noheader > gpurun_out/fl9_box.txt
for i in 1 2 3; do
  for v in ALT_TC_ROUND=0 ALT_TC_ROUND=1; do
    env $v python -m pytest tests/test_gpu_conv3d.py tests/test_gpu_conv.py tests/test_gpu_store_at.py -q --timeout 900 -p no:cacheprovider > gpurun_out/fl9_${v}_$i.txt 2>&1
  done
done
