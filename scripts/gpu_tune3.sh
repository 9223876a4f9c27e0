#!/bin/bash
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/tune
make -C paper_conf_eurosys_xuxpwwwdxcwc23_b200 -j8 >/dev/null 2>&1
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -2
rm -f tune_cache.jsonl chain_tune.json
timeout 1200 python scripts/tune_r50.py 32 gpurun_out/tune/tune_cache.jsonl 2>&1 | grep -v "Exception\|Traceback\|File \|AttributeError" | cut -c1-140
timeout 1500 python scripts/tune_chains.py gpurun_out/tune/chain_tune.json 2>&1 | grep -v "Exception\|Traceback\|File \|AttributeError" | tail -3
for w in r50 r18 mv2; do timeout 300 python bench.py --workload $w --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('$w', d['value'], d['ms_per_step'], [l['us'] for l in d.get('per_layer', [])])"; done
