#!/bin/bash
cd $GRAFT_REPO_ROOT
for v in e8 e16; do
  echo "== $v"
  ALT_LIB_VARIANT=$v timeout 300 python scripts/diag4.py 2>&1 | grep "^N="
  for w in r50 r18 mv2; do ALT_LIB_VARIANT=$v timeout 300 python bench.py --workload $w --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('$w', d['value'], d['ms_per_step'], [l['us'] for l in d.get('per_layer', [])])"; done
done
ALT_LIB_VARIANT=e16 timeout 600 python -m pytest tests -m gpu -x -q 2>&1 | tail -2
