cd $GRAFT_REPO_ROOT
timeout 600 python -m pytest tests/test_gpu_conv.py -q -k "tc_" -x 2>&1 | tail -30 > gpurun_out/tc1.txt
timeout 600 python -m pytest tests/test_gpu_conv.py -q -k "tc_" 2>&1 | grep -E "passed|failed|FAILED|Error" | tail -30 >> gpurun_out/tc1.txt
cat gpurun_out/tc1.txt | tail -40
