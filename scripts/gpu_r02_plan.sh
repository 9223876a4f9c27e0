# after the topological X0 rule: chain tests, shard tests, chain bench lines
python -m pytest tests/test_gpu_chain.py tests/test_gpu_fullsize.py tests/test_gpu_dist.py -q -p no:cacheprovider --timeout 1500 > gpurun_out/plan_pytest.txt 2>&1; echo "rc=$?" >> gpurun_out/plan_pytest.txt
python bench.py --workload r18 --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/plan_r18.json 2>/dev/null
python bench.py --workload mv2 --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/plan_mv2.json 2>/dev/null
