# re-tune the ResNet-50 b32 and b1 layer sets on the current kernel, then A/B the bench line
cp tune_cache.jsonl gpurun_out/tune_cache_old.jsonl
python bench.py --steps 10 --warmup 3 --no-aux --no-cpu-baseline > gpurun_out/rt_old.json 2>/dev/null
python scripts/tune_r50.py 32 > gpurun_out/rt_log32.txt 2>&1
python scripts/tune_r50.py 1 > gpurun_out/rt_log1.txt 2>&1
cp tune_cache.jsonl gpurun_out/tune_cache_new.jsonl
python bench.py --steps 10 --warmup 3 --no-aux --no-cpu-baseline > gpurun_out/rt_new.json 2>/dev/null
python bench.py --batch 1 --steps 10 --warmup 3 --no-aux --no-cpu-baseline > gpurun_out/rt_new_b1.json 2>/dev/null
cp gpurun_out/tune_cache_old.jsonl tune_cache.jsonl
python bench.py --steps 10 --warmup 3 --no-aux --no-cpu-baseline > gpurun_out/rt_old2.json 2>/dev/null
python bench.py --batch 1 --steps 10 --warmup 3 --no-aux --no-cpu-baseline > gpurun_out/rt_old_b1.json 2>/dev/null
