#!/bin/bash
cd $GRAFT_REPO_ROOT
make -C paper_conf_eurosys_xuxpwwwdxcwc23_b200 -j8 >/dev/null 2>&1
timeout 600 python -m pytest tests/test_gpu_relayout.py -x -q 2>&1 | tail -2
timeout 300 python scripts/chain_ops.py mv2 16 2>/dev/null | grep -v "^Exception\|^Traceback\|^  File\|^Attribute" | cut -c1-90
timeout 300 python bench.py --workload relayout --no-cpu-baseline 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('relayout', d['value'])
for c in d['cases']:
    if c['case'].startswith('R7'): print('  ', c)"
