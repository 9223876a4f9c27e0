#!/bin/bash
# bisect the pytest sequence that makes the first store_at TC GEMM launch lose its residual
run() { ALT_FLAKE_DIAG=1 python -m pytest $1 -q --timeout 900 -p no:cacheprovider -k "$2" > gpurun_out/fl3_$3.txt 2>&1; }
run "tests/test_gpu_store_at.py" "parity" a
run "tests/test_gpu_fullsize.py tests/test_gpu_store_at.py" "b1_tuned or matmul_store_at_parity" b
run "tests/test_gpu_fullsize.py tests/test_gpu_store_at.py" "b1_tuned or 384x192x256p7tc-bf16" c
run "tests/test_gpu_store_at.py" "" d
run "tests/test_gpu_fullsize.py tests/test_gpu_store_at.py" "b1_tuned or parity" e
