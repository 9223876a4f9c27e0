#!/bin/bash
cd $GRAFT_REPO_ROOT
make -C paper_conf_eurosys_xuxpwwwdxcwc23_b200 -j8 >/dev/null 2>&1
timeout 600 python -m pytest tests -m gpu -x -q 2>&1 | tail -2
for w in mv2 r18 r50; do timeout 300 python bench.py --workload $w --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('$w', d['value'], d['ms_per_step'])"; done
