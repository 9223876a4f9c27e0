#!/bin/bash
make -C paper_conf_eurosys_xuxpwwwdxcwc23_b200 -j8 >/dev/null 2>&1
timeout 600 python -m pytest tests/test_gpu_conv.py tests/test_gpu_chain.py -q -x 2>&1 | tail -3
timeout 600 python scripts/exp_epi.py 2>&1 | grep "tiles/cta=32"
timeout 300 python bench.py --steps 20 --warmup 3 --no-cpu-baseline 2>&1 | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); print(d['value'], d['ms_per_step']); [print(l) for l in d['per_layer']]"
