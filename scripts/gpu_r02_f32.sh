python scripts/f32_error_scaling.py > gpurun_out/f32err.txt 2>&1
python -m pytest tests/test_gpu_fp32tc.py -q --timeout 600 -p no:cacheprovider > gpurun_out/f32.txt 2>&1; echo "rc=$?" >> gpurun_out/f32.txt
