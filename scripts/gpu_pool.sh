#!/bin/bash
cd $GRAFT_REPO_ROOT
make -C paper_conf_eurosys_xuxpwwwdxcwc23_b200 -j8 >/dev/null 2>&1
timeout 600 python -m pytest tests -m gpu -q -k "pool or resnet18 or chain" 2>&1 | tail -2
timeout 300 ncu --metrics gpu__time_duration.sum -k regex:k_pool -c 1 python scripts/prof_hbm_ops.py 2>&1 | grep -E "gpu__time"
timeout 300 python bench.py --workload r18 --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('r18', d['value'], d['ms_per_step'])"
