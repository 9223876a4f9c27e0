#!/bin/bash
cd $GRAFT_REPO_ROOT
make -C paper_conf_eurosys_xuxpwwwdxcwc23_b200 -j8 >/dev/null 2>&1
timeout 600 python -m pytest tests -m gpu -x -q -k "depthwise or mobilenet or dw" 2>&1 | tail -2
for f in 0 1; do ALT_DW_FORM=$f timeout 300 python bench.py --workload mv2 --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('form $f mv2', d['value'], d['ms_per_step'])"; done
timeout 300 ncu --metrics gpu__time_duration.sum -k regex:k_dw -c 6 python scripts/prof_hbm_ops.py 2>&1 | grep -E "k_dw|gpu__time" | head -8
ALT_DW_FORM=0 timeout 300 ncu --metrics gpu__time_duration.sum -k regex:k_dw -c 6 python scripts/prof_hbm_ops.py 2>&1 | grep -E "k_dw|gpu__time" | head -8
