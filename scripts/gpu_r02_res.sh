# resident-B conv + K_WIN relayout: parity, then A/B timings
python -m pytest tests/test_gpu_relayout.py -q -x -p no:cacheprovider > gpurun_out/rl_pytest.txt 2>&1; echo "rc=$?" >> gpurun_out/rl_pytest.txt
python -m pytest tests -m gpu -q -x -p no:cacheprovider --timeout 1500 --deselect tests/test_gpu_relayout.py > gpurun_out/res_pytest.txt 2>&1; echo "rc=$?" >> gpurun_out/res_pytest.txt
python bench.py --workload relayout --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/rl_new.json 2> gpurun_out/rl_new.err
ALT_WIN_BUDGET=110000 python bench.py --workload relayout --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/rl_b110.json 2> gpurun_out/rl_b110.err
python bench.py --steps 10 --warmup 3 --no-aux --no-cpu-baseline > gpurun_out/r50_res.json 2> gpurun_out/r50_res.err
ALT_TC_NO_BRES=1 python bench.py --steps 10 --warmup 3 --no-aux --no-cpu-baseline > gpurun_out/r50_nores.json 2> gpurun_out/r50_nores.err
python bench.py --workload r18 --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/r18_res.json 2> gpurun_out/r18_res.err
ALT_TC_NO_BRES=1 python bench.py --workload r18 --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/r18_nores.json 2> gpurun_out/r18_nores.err
python bench.py --workload mv2 --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/mv2_res.json 2> gpurun_out/mv2_res.err
ALT_TC_NO_BRES=1 python bench.py --workload mv2 --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/mv2_nores.json 2> gpurun_out/mv2_nores.err
