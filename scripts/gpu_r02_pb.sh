python -m pytest tests/test_gpu_relayout.py -q -x -p no:cacheprovider > gpurun_out/rl_pytest.txt 2>&1; echo "rc=$?" >> gpurun_out/rl_pytest.txt
python scripts/relayout_probe.py R7 R5 R6 > gpurun_out/pb_probe.txt 2>&1
ALT_PB_NOSWZ=1 python scripts/relayout_probe.py R7 >> gpurun_out/pb_probe.txt 2>&1
