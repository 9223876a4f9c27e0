# relayout: K_WIN transposed stage, budget A/B, parity
python -m pytest tests/test_gpu_relayout.py -q -x -p no:cacheprovider > gpurun_out/rl_pytest.txt 2>&1; echo "rc=$?" >> gpurun_out/rl_pytest.txt
python bench.py --workload relayout --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/rl_new.json 2> gpurun_out/rl_new.err
ALT_WIN_BUDGET=110000 python bench.py --workload relayout --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/rl_b110.json 2> gpurun_out/rl_b110.err
ALT_WIN_BUDGET=24000 python bench.py --workload relayout --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/rl_b24.json 2> gpurun_out/rl_b24.err
ALT_RELAYOUT_NOWIN=1 python bench.py --workload relayout --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/rl_old.json 2> gpurun_out/rl_old.err
