#!/bin/bash
cd $GRAFT_REPO_ROOT
for v in "" dw3; do
  echo "== variant '$v'"
  ALT_LIB_VARIANT=$v timeout 300 ncu --metrics gpu__time_duration.sum -k regex:k_dw -c 1 python scripts/prof_hbm_ops.py 2>&1 | grep -E "gpu__time"
  ALT_LIB_VARIANT=$v timeout 300 python bench.py --workload mv2 --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('mv2', d['value'], d['ms_per_step'])"
done
