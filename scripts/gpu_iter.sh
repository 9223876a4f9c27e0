#!/bin/bash
# quick iteration: build, GPU parity tests, chain per-op timing, R50 bench line
cd $GRAFT_REPO_ROOT; O=gpurun_out/iter; mkdir -p $O
make -C paper_conf_eurosys_xuxpwwwdxcwc23_b200 -j8 >/dev/null 2>&1 || { echo build failed; exit 1; }
timeout 900 python -m pytest tests -m gpu -x -q > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -15 $O/pytest_gpu.log
timeout 300 python scripts/chain_ops.py mv2 16 2>/dev/null | grep -v "^Exception\|^Traceback\|^  File\|^Attribute" > $O/mv2_ops.txt; tail -1 $O/mv2_ops.txt
timeout 300 python scripts/chain_ops.py r18 256 2>/dev/null | grep -v "^Exception\|^Traceback\|^  File\|^Attribute" > $O/r18_ops.txt; cut -c1-60 $O/r18_ops.txt
for w in r18 mv2; do timeout 300 python bench.py --workload $w --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('$w', d['value'], d['ms_per_step'])"; done
timeout 300 python bench.py --no-cpu-baseline > $O/bench.json 2>/dev/null; python -c "import json; d=json.loads(open('$O/bench.json').read().strip().splitlines()[-1]); print('r50', d['value'], d['ms_per_step'])"
timeout 300 python bench.py --workload relayout --no-cpu-baseline 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('relayout', d['value'])
for c in d['cases']: print('  ', c)"
python -c "import json; d=json.loads(open('$O/bench.json').read().strip().splitlines()[-1]); [print(l) for l in d['per_layer']]"
