#!/bin/bash
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 900 python scripts/cfg_sweep.py 2>&1 | grep -v "^Exception ignored\|__del__\|AttributeError\|Traceback" | tee gpurun_out/s2j_sweep.txt
