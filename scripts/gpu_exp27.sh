#!/bin/bash
make -C paper_conf_eurosys_xuxpwwwdxcwc23_b200 -j8 >/dev/null 2>&1
timeout 900 python -m pytest tests/ -m gpu -q -x 2>&1 | tail -3
ALT_TC_STORE=tma timeout 900 python -m pytest tests/test_gpu_conv.py -m gpu -q -x 2>&1 | tail -2
for m in tma direct; do
echo "== $m"
ALT_TC_STORE=$m EPI_K=64,256 timeout 300 python scripts/exp_epi.py 2>&1
ALT_TC_STORE=$m timeout 300 python bench.py --steps 20 --warmup 3 --no-cpu-baseline 2>&1 | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); print(d['value'], d['ms_per_step']); [print(l['layer'], l['us'], l['tflops']) for l in d['per_layer']]"
done
