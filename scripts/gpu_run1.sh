cd $GRAFT_REPO_ROOT
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/smi.txt 2>&1
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -40 > gpurun_out/gpu_tests1.txt
timeout 300 python __graft_entry__.py > gpurun_out/smoke1.txt 2>&1
tail -5 gpurun_out/gpu_tests1.txt
