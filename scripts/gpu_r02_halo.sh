python scripts/tune_halo_r50.py 32 gpurun_out/tune_cache.jsonl > gpurun_out/tune_halo32.txt 2>&1
python scripts/tune_halo_r50.py 1 gpurun_out/tune_cache.jsonl > gpurun_out/tune_halo1.txt 2>&1
python -m pytest tests/test_gpu_chain.py -q -k tune --timeout 600 -p no:cacheprovider > gpurun_out/t4.txt 2>&1
