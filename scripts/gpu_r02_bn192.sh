# single-CTA BLOCK_N 192: parity, BERT re-tune with it, bench before / after
python -m pytest tests/test_gpu_conv.py -q -p no:cacheprovider -k "192 or tail_split or block_n" > gpurun_out/bn192_pytest.txt 2>&1; echo "rc=$?" >> gpurun_out/bn192_pytest.txt
python bench.py --workload bert --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bn192_bert_old.json 2>/dev/null
python scripts/tune_bert.py gpurun_out/tune_cache_bn192.jsonl > gpurun_out/bn192_tune_log.txt 2>&1
python bench.py --workload bert --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bn192_bert_new.json 2>/dev/null
