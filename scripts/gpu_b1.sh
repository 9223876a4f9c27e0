#!/bin/bash
# BASELINE config 2 at batch 1: tune the layer set at N = 1, then the bench line
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/b1
make -C paper_conf_eurosys_xuxpwwwdxcwc23_b200 -j8 >/dev/null 2>&1
timeout 1500 python scripts/tune_r50.py 1 gpurun_out/b1/tune_cache.jsonl 2>&1 | grep -v "Exception\|Traceback\|File \|AttributeError" | cut -c1-120 | tail -4
timeout 300 python bench.py --batch 1 --no-cpu-baseline > gpurun_out/b1/bench_b1.json 2>/dev/null
python -c "import json; d=json.loads(open('gpurun_out/b1/bench_b1.json').read().strip().splitlines()[-1]); print('b1', d['value'], d['ms_per_step'], d['roofline']['set_roofline_time_frac'], [l['us'] for l in d['per_layer']])"
