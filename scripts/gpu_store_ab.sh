#!/bin/bash
cd $GRAFT_REPO_ROOT
make -C paper_conf_eurosys_xuxpwwwdxcwc23_b200 -j8 >/dev/null 2>&1
for m in t d; do
  for w in r50 r18 mv2; do ALT_TC_STORE=$m timeout 300 python bench.py --workload $w --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('$m $w', d['value'], d['ms_per_step'], [l['us'] for l in d.get('per_layer', [])])"; done
done
