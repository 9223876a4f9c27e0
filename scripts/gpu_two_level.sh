#!/bin/bash
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/tune2
make -C paper_conf_eurosys_xuxpwwwdxcwc23_b200 -j8 >/dev/null 2>&1
timeout 300 python bench.py --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('r50 before', d['value'], d['ms_per_step'])"
timeout 1800 python scripts/tune_two_level.py 32 gpurun_out/tune2/tune_cache.jsonl 2>&1 | grep -v "Exception\|Traceback\|File \|AttributeError"
timeout 300 python bench.py --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('r50 after', d['value'], d['ms_per_step'], [l['us'] for l in d['per_layer']])"
timeout 600 python -m pytest tests/test_gpu_fullsize.py -q -k r50 2>&1 | tail -2
