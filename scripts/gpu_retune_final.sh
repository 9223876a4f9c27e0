#!/bin/bash
# re-tune (R50 b32 + b1, chains), then the round evidence run
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/tune
make -C paper_conf_eurosys_xuxpwwwdxcwc23_b200 -j8 >/dev/null 2>&1
timeout 1500 python scripts/tune_r50.py 32 > /dev/null 2>&1
timeout 1500 python scripts/tune_r50.py 1 gpurun_out/tune/tune_cache.jsonl > /dev/null 2>&1
timeout 1500 python scripts/tune_chains.py gpurun_out/tune/chain_tune.json > /dev/null 2>&1
timeout 1500 python scripts/tune_r18_shards.py gpurun_out/tune/chain_tune.json 2>&1 | grep "r18 per-GPU"
bash scripts/gpu_r01_full.sh
