#!/bin/bash
# A/B of the R50 bench between libalt_head.so (last commit) and the working tree's libalt.so
cd $GRAFT_REPO_ROOT
for r in 1 2; do
for v in head ""; do
  ALT_LIB_VARIANT=$v timeout 300 python bench.py --no-cpu-baseline --steps 20 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('variant=${v:-cur}', d['value'], d['ms_per_step'], [l['us'] for l in d['per_layer']])"
done; done
