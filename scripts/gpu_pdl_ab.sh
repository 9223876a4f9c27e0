#!/bin/bash
cd $GRAFT_REPO_ROOT
for env in "X=1" "ALT_PDL=0 ALT_PDL_CC=0"; do
  for w in mv2 r50; do env $env timeout 300 python bench.py --workload $w --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('$env $w', d['value'], d['ms_per_step'])"; done
done
