# re-tune the chain loop schedules (MV2 b16 / b1, R18 b256 and its shards) and the BERT GEMMs on the
# current kernel; bench lines before / after
python bench.py --steps 10 --warmup 3 --no-aux --no-cpu-baseline > gpurun_out/rt2_r50_merged.json 2>/dev/null
python bench.py --workload r18 --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/rt2_r18_old.json 2>/dev/null
python bench.py --workload mv2 --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/rt2_mv2_old.json 2>/dev/null
python bench.py --workload bert --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/rt2_bert_old.json 2>/dev/null
python scripts/tune_chains.py gpurun_out/chain_tune_new.json > gpurun_out/rt2_chains_log.txt 2>&1
python scripts/tune_r18_shards.py gpurun_out/chain_tune_new.json 128 64 32 > gpurun_out/rt2_shards_log.txt 2>&1
python scripts/tune_bert.py gpurun_out/tune_cache_bert.jsonl > gpurun_out/rt2_bert_log.txt 2>&1
python bench.py --workload r18 --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/rt2_r18_new.json 2>/dev/null
python bench.py --workload mv2 --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/rt2_mv2_new.json 2>/dev/null
python bench.py --workload bert --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/rt2_bert_new.json 2>/dev/null
