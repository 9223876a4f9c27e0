#!/bin/bash
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/ -m gpu -q -x 2>&1 | tail -5 > gpurun_out/s2a_tests.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/s2a_smoke.txt 2>&1
timeout 600 python bench.py > gpurun_out/s2a_bench.json 2> gpurun_out/s2a_bench.err
timeout 300 python bench.py --steps 20 --warmup 3 --no-cpu-baseline --eager > gpurun_out/s2a_bench_eager.json 2>>gpurun_out/s2a_bench.err
cat gpurun_out/s2a_tests.txt gpurun_out/s2a_smoke.txt
python -c "
import json; d=json.loads(open('gpurun_out/s2a_bench.json').read().strip().splitlines()[-1])
for l in d.pop('per_layer',[]): print(l)
print(json.dumps(d))
"
tail -3 gpurun_out/s2a_bench.err
