#!/bin/bash
make -C paper_conf_eurosys_xuxpwwwdxcwc23_b200 -j8 >/dev/null 2>&1
timeout 600 python -m pytest tests/test_gpu_conv.py tests/test_gpu_chain.py tests/test_gpu_relayout.py -q -x 2>&1 | tail -5
timeout 300 python bench.py --workload relayout --steps 10 --warmup 3 | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); print(d['value']); [print(c) for c in d['cases']]"
timeout 300 python bench.py --workload r18 --steps 10 --warmup 3 | tail -1 | cut -c1-300
timeout 300 python bench.py --workload mv2 --steps 10 --warmup 3 | tail -1 | cut -c1-300
