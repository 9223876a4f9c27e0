#!/bin/bash
# A/B: bench value for several library variants / env settings, interleaved
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
run() { env "$@" timeout 300 python bench.py --steps 20 --warmup 3 --no-cpu-baseline 2>/dev/null | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); print('$*', d['value'], d['ms_per_step'])"; }
for rep in 1 2; do
  for v in "$@"; do run $v; done
done
