#!/bin/bash
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 900 python -m pytest tests/ -m gpu -q -x 2>&1 | tail -2
timeout 300 python bench.py --steps 20 --warmup 3 --no-cpu-baseline 2>&1 | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); print(d['value'], d['ms_per_step'], d['roofline']['achieved']); [print(l['layer'], l['us'], l['tflops'], l['block_n']) for l in d['per_layer']]"
make -C paper_conf_eurosys_xuxpwwwdxcwc23_b200 clean >/dev/null
make -C paper_conf_eurosys_xuxpwwwdxcwc23_b200 -j8 EXTRA=-DALT_DBG_TILE=2 >/dev/null 2>&1
timeout 300 python scripts/exp_dbg5.py l1.1x1a 2>&1 | grep -v "Exception ignored\|Traceback\|__del__\|AttributeError"
timeout 300 python scripts/exp_dbg5.py l4.1x1b 2>&1 | grep -v "Exception ignored\|Traceback\|__del__\|AttributeError"
make -C paper_conf_eurosys_xuxpwwwdxcwc23_b200 clean >/dev/null
