python scripts/epi_probe.py > gpurun_out/epi_round.txt 2>&1
ALT_TC_ROUND=0 python scripts/epi_probe.py > gpurun_out/epi_warp.txt 2>&1
python -m pytest tests/test_gpu_conv.py tests/test_gpu_mnmajor.py tests/test_gpu_fp32tc.py tests/test_gpu_chain.py -q -x --timeout 900 -p no:cacheprovider > gpurun_out/conv.txt 2>&1; echo "rc=$?" >> gpurun_out/conv.txt
